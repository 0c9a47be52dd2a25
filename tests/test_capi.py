"""CPU checks of the C ABI: libgtr.so loads and exports every symbol
include/gtr.h declares; host-only calls work without a GPU."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "gtr.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gtr_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    from paper_conf_cgo_hubercgtddcd22_b200 import gtr
    lib = ctypes.CDLL(gtr.LIB_PATH)
    syms = declared_symbols()
    assert len(syms) >= 15
    for s in syms:
        assert hasattr(lib, s), s
    assert set(syms) == set(gtr.EXPORTED)


def test_host_only_calls():
    from paper_conf_cgo_hubercgtddcd22_b200 import gtr
    assert gtr.gtr_version() == 1000
    assert "heap" in gtr.gtr_strerror(gtr.GTR_EHEAP)
    # energies + one i32 column minimum per (4096 union points, nuclide)
    total = 355 * 11303
    assert gtr.gtr_xs_build_workspace_bytes(355, 11303) == total * 8 + -(-total // 4096) * 355 * 4
    # sorted mode: two 16-byte records + a key per lookup, 12 x 2^17 bins + block totals
    assert gtr.gtr_xs_sorted_workspace_bytes(17_000_000) == 36 * 17_000_000 + 4 * (12 * 2**17 + 12 * 2**17 // 1024)


def test_library_is_sm100a():
    import subprocess
    from paper_conf_cgo_hubercgtddcd22_b200 import gtr
    r = subprocess.run(["cuobjdump", "--list-elf", gtr.LIB_PATH], capture_output=True, text=True)
    assert r.returncode == 0
    assert "sm_100a" in r.stdout


def test_oracle_is_not_reachable_from_product():
    pkg = os.path.join(ROOT, "paper_conf_cgo_hubercgtddcd22_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.h" not in txt and "liboracle" not in txt, f


def test_product_fails_loudly_without_library():
    """No CPU fallback: with the CUDA library absent the binding refuses to import."""
    import subprocess
    import sys
    env = dict(os.environ, GTR_LIB=os.path.join(ROOT, "build", "does_not_exist", "libgtr.so"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_cgo_hubercgtddcd22_b200.gtr"],
                       cwd=ROOT, env=env, capture_output=True, text=True)
    assert r.returncode != 0
    assert "ImportError" in r.stderr and "no CPU fallback" in r.stderr
