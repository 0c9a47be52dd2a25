"""Build exp/libgtr_head.so: the default build's objects with the CSM+SPMD
XS group unit (thread_limit 256) compiled from the committed HEAD sources --
an A/B baseline for uncommitted kernel edits (load with GTR_LIB=...)."""
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_hubercgtddcd22_b200 import build as B  # noqa: E402

src = "/tmp/gtr_head_src"
subprocess.check_call(["rm", "-rf", src])
os.makedirs(src)
subprocess.check_call(f"git -C {ROOT} archive HEAD paper_conf_cgo_hubercgtddcd22_b200/csrc include | tar -x -C {src}",
                      shell=True)
B.build(verbose=False)
objs = [o for o in sorted(glob.glob(os.path.join(B.OBJ, "*.o"))) if not os.path.basename(o).startswith("xs_grp_t256.")]
os.makedirs(os.path.join(ROOT, "exp"), exist_ok=True)
o = os.path.join(ROOT, "exp", "xs_grp_t256_head.o")
fl = [f for f in B.CFLAGS if not f.startswith("-I")] + ["-I" + os.path.join(src, "include")]
subprocess.check_call([B.NVCC] + fl + ["-DGTR_V_GROUP_NT=256", "-c",
                       os.path.join(src, "paper_conf_cgo_hubercgtddcd22_b200", "csrc", "xs_variant.cu"), "-o", o])
subprocess.check_call([B.NVCC] + B.ARCH + ["-shared", "-o", os.path.join(ROOT, "exp", "libgtr_head.so")] + objs + [o])
print(os.path.join(ROOT, "exp", "libgtr_head.so"))
