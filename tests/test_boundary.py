"""CPU-side checks of the C-ABI boundary: the library loads, exports every symbol include/abft.h
declares, validates arguments before touching the device, and the Python binding marshals the
same struct layouts as the header (no compute calls: no GPU here)."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "abft.h")


def declared_functions():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:int|int64_t|const char\*)\s+(abft_\w+)\s*\(", txt, flags=re.M)))


def test_header_declares_the_survey_boundary():
    names = declared_functions()
    for must in ("abft_potrf", "abft_encode", "abft_verify", "abft_potrf_ex", "abft_potrf_dist",
                 "abft_nccl_id", "abft_comm_init"):
        assert must in names


def test_library_exports_every_declared_symbol():
    import paper_conf_ipps_chenlc16_b200 as p
    lib = ctypes.CDLL(p.LIB_PATH)
    for name in declared_functions():
        assert hasattr(lib, name), name
    assert set(declared_functions()) <= set(p.EXPORTS)
    assert "sm_100a" in p.abft_version()


def test_struct_layouts_match_header():
    import paper_conf_ipps_chenlc16_b200 as p
    import synthetic as syn
    assert ctypes.sizeof(p.Event) == 48 == p.EVENT_DTYPE.itemsize
    assert p.INJ_DTYPE.itemsize == 48 == syn.INJ_DTYPE.itemsize
    assert ctypes.sizeof(p.Report) == 14 * 8
    assert ctypes.sizeof(p.Options) == 40


def test_sm100a_code_in_library():
    import subprocess
    import paper_conf_ipps_chenlc16_b200 as p
    out = subprocess.run(["cuobjdump", "-sass", p.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "DMMA.8x8x4" in out          # FP64 tensor-core path of the GEMM kernels
    assert "LDGSTS" in out              # cp.async staging


@pytest.mark.parametrize("args,expect", [
    ((-1, 32, 1, 1), -1),           # n < 0
    ((64, 0, 1, 64), -2),           # nb < 1
    ((64, 24, 1, 64), -2),          # n % nb != 0 (version-1 restriction)
    ((64, 32, 0, 64), -3),          # A == NULL
    ((64, 32, 1, 63), -4),          # lda < n
])
def test_argument_errors_before_any_device_work(args, expect):
    import paper_conf_ipps_chenlc16_b200 as p
    n, nb, A, lda = args
    assert p.lib().abft_potrf(n, nb, A, lda, None, None, None) == expect


def test_injection_validation():
    import paper_conf_ipps_chenlc16_b200 as p
    import synthetic as syn
    bad = [dict(k=0, hook="REST", row=3, col=5, bit=1),                 # upper triangle
           dict(k=1, hook="POTRF_OUT", row=70, col=0, bit=1),           # outside tile (1,1)
           dict(k=0, hook="TRSM_OUT", row=10, col=10, bit=1),           # not in panel 0
           dict(k=2, hook="UPDATE_OUT", row=200, col=10, bit=1),        # not trailing
           dict(k=0, hook="REST", target="CHK", row=0, col=100, bit=1),  # chk of an upper tile
           dict(k=9, hook="REST", row=3, col=1, bit=1)]                 # k > N
    for spec in bad:
        arr = syn.inj_array([spec])
        st = p.lib().abft_potrf(256, 64, 1, 256, None, arr.ctypes.data, None)
        assert st == -6, spec


def test_binding_refuses_missing_library(tmp_path):
    """The product path has no CPU fallback: without libabft.so the import fails loudly."""
    import subprocess
    import sys
    import shutil
    pkg = tmp_path / "paper_conf_ipps_chenlc16_b200"
    shutil.copytree(os.path.join(ROOT, "paper_conf_ipps_chenlc16_b200"), pkg,
                    ignore=shutil.ignore_patterns("*.so", "csrc"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_ipps_chenlc16_b200"], cwd=tmp_path,
                       capture_output=True, text=True)
    assert r.returncode != 0 and "no CPU fallback" in r.stderr


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_chenlc16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "oracle/" not in txt and "liboracle" not in txt, f
    # and the oracle never includes the product
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "import paper_conf_ipps_chenlc16_b200" not in txt and "libabft" not in txt, f
