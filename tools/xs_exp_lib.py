"""Experiment libraries for the XS lookup kernel: recompile only the CSM+SPMD
group units of xs_variant.cu with extra defines and link them with the default
build's other objects into exp/libgtr_<name>.so (load with GTR_LIB=...).

    python tools/xs_exp_lib.py NAME NT -DGTR_XS_MINB=3 [...]   (NT: 128 or 256)
    GTR_EXP_FAMILY=rs python tools/xs_exp_lib.py NAME 128 -DGTR_RS_MINB=5
"""
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_hubercgtddcd22_b200 import build as B  # noqa: E402


def main():
    name, nt_exp, defs = sys.argv[1], int(sys.argv[2]), sys.argv[3:]
    fam = os.environ.get("GTR_EXP_FAMILY", "xs")
    B.build(verbose=False)
    out_dir = os.path.join(ROOT, "exp")
    os.makedirs(out_dir, exist_ok=True)
    objs = []
    for o in sorted(glob.glob(os.path.join(B.OBJ, "*.o"))):
        base = os.path.basename(o)
        if base.startswith(f"{fam}_grp_t{nt_exp}."):
            continue
        objs.append(o)
    for nt in (nt_exp,):
        o = os.path.join(out_dir, f"{fam}_grp_t{nt}_{name}.o")
        fl = B.CFLAGS if fam != "rs" else ["-fmad=true" if f == "-fmad=false" else f for f in B.CFLAGS]
        cmd = [B.NVCC] + fl + [f"-DGTR_V_GROUP_NT={nt}"] + defs + [
            "-Xptxas", "-v", "-c", os.path.join(B.CSRC, fam + "_variant.cu"), "-o", o]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode:
            sys.exit(r.stderr)
        lines = r.stderr.splitlines()
        for i, l in enumerate(lines):
            if "Cfg<3, 3, true" in l or "ILi3ELi3ELb1E" in l and "Function properties" in l:
                print(nt, lines[i + 1].strip(), "|", lines[i + 2].strip())
        objs.append(o)
    lib = os.path.join(out_dir, f"libgtr_{name}.so")
    subprocess.check_call([B.NVCC] + B.ARCH + ["-shared", "-o", lib] + objs)
    print(lib)


if __name__ == "__main__":
    main()
