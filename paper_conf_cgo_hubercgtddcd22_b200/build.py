"""Build libgtr.so in-tree: every CUDA translation unit for sm_100a.

GENERIC and GENERIC_CASCADE kernels make indirect calls, and ptxas assumes an
indirect call may reach every address-taken function of the module (the
"spurious call edges" of PAPER.md:593-597, fn. 4) -- inheriting their
registers and even their static shared memory.  Each application in the paper
is its own module, so each GENERIC/CASCADE variant is compiled as its own
translation unit here; CSM and SPMD variants (no function pointers) are
grouped per thread_limit.  Objects are cached under build/ by flags + the mtime of the source and
the headers it includes.

    python -m paper_conf_cgo_hubercgtddcd22_b200.build [-j N] [--force]
"""
import argparse
import hashlib
import os
import re
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
ROOT = os.path.dirname(PKG)
OBJ = os.path.join(ROOT, "build", "obj")
LIB = os.environ.get("GTR_LIB_OUT", os.path.join(PKG, "libgtr.so"))

NVCC = os.environ.get("NVCC", shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ARCH + ["-O3", "-std=c++17", "-lineinfo", "-fmad=false", "-Xfatbin=-compress-all", "-Xcompiler", "-fPIC",
                 "-Xcompiler", "-O2", "-I" + os.path.join(ROOT, "include")]
CFLAGS += os.environ.get("GTR_NVCC_EXTRA", "").split()   # experiments only

# family -> (thread_limits, SPMD-only flag variants)
FAMILIES = {
    "xs": ([128, 256], []),
    "fj": ([32, 128, 256, 512], [1]),      # GTR_F_BCAST_1BAR
    "sem": ([64, 128], [2]),               # GTR_F_SEPARATE_GUARDS
    "su3": ([64, 128], []),
    "rs": ([128], []),                     # 256: static-shared placement exceeds 48 KB
}
COMMON = ["capi.cu", "xs.cu", "fj.cu", "sem.cu", "su3.cu", "rs.cu"]


def units():
    """(object name, source, extra defines) for every translation unit."""
    out = [(os.path.splitext(s)[0], s, []) for s in COMMON]
    for fam, (nts, flagvars) in FAMILIES.items():
        src = fam + "_variant.cu"
        for nt in nts:
            for mode in (0, 1):
                for pl in range(5):
                    for fold in (0, 1):
                        out.append((f"{fam}_m{mode}_p{pl}_f{fold}_t{nt}", src,
                                    [f"-DGTR_V_MODE={mode}", f"-DGTR_V_PL={pl}",
                                     f"-DGTR_V_FOLD={fold}", f"-DGTR_V_NT={nt}"]))
            out.append((f"{fam}_grp_t{nt}", src, [f"-DGTR_V_GROUP_NT={nt}"]))
            for fl in flagvars:
                out.append((f"{fam}_spmd_t{nt}_fl{fl}", src,
                            [f"-DGTR_V_GROUP_NT={nt}", f"-DGTR_V_FLAGS={fl}", "-DGTR_V_SPMD_ONLY"]))
    return out


_INC = re.compile(r'^\s*#\s*include\s+"([^"]+)"', re.M)


def _deps_mtime(src, seen=None):
    """Newest mtime of `src` and every file it #includes with quotes (recursively)."""
    seen = set() if seen is None else seen
    path = os.path.normpath(src if os.path.isabs(src) else os.path.join(CSRC, src))
    if path in seen or not os.path.exists(path):
        return 0.0
    seen.add(path)
    m = os.path.getmtime(path)
    with open(path) as f:
        for inc in _INC.findall(f.read()):
            m = max(m, _deps_mtime(os.path.join(os.path.dirname(path), inc), seen))
    return m


def _compile(job, force):
    name, src, defs = job
    deps_m = _deps_mtime(src)
    flags = CFLAGS + defs
    if src.startswith("rs"):
        # RS parity is within a tolerance (libm sin/cos/atan differ anyway,
        # DESIGN.md R-RS-tol): its TUs may contract a*b+c into fp64 FMAs.
        # XS and SU3 stay -fmad=false: bit-identical to the oracle.
        flags = ["-fmad=true" if f == "-fmad=false" else f for f in flags]
    key = hashlib.sha1((" ".join(flags) + src).encode()).hexdigest()[:10]
    obj = os.path.join(OBJ, f"{name}.{key}.o")
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= deps_m:
        return obj, None
    cmd = [NVCC] + flags + ["-c", os.path.join(CSRC, src), "-o", obj + ".tmp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        return None, f"{name}: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}"
    os.replace(obj + ".tmp", obj)
    return obj, None


def build(jobs=None, force=False, verbose=True):
    os.makedirs(OBJ, exist_ok=True)
    us = units()
    jobs = jobs or max(1, os.cpu_count() or 1)
    with ThreadPoolExecutor(jobs) as ex:
        res = list(ex.map(lambda j: _compile(j, force), us))
    errs = [e for _, e in res if e]
    if errs:
        raise RuntimeError("nvcc failed:\n" + "\n".join(errs[:3]))
    objs = [o for o, _ in res]
    if (not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= max(os.path.getmtime(o) for o in objs)):
        return LIB
    cmd = [NVCC] + ARCH + ["-shared", "-Xlinker", "-z", "-Xlinker", "defs", "-o", LIB + ".tmp"] + objs
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    # drop stale objects of older flag sets (default build only)
    if not os.environ.get("GTR_NVCC_EXTRA"):
        keep = set(os.path.basename(o) for o in objs)
        for f in os.listdir(OBJ):
            if f.endswith(".o") and f not in keep:
                os.remove(os.path.join(OBJ, f))
    if verbose:
        print(f"built {LIB} from {len(objs)} translation units")
    return LIB


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=None)
    ap.add_argument("--force", action="store_true")
    a = ap.parse_args()
    try:
        build(a.j, a.force)
    except RuntimeError as e:
        print(e, file=sys.stderr)
        sys.exit(1)
