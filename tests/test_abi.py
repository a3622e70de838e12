"""CPU checks of the boundary: libdysel.so builds, loads and exports every
function include/dysel.h declares (no compute calls without a GPU)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "dysel.h")


def declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dysel_[a-z0-9_]+)\s*\(", src)) - {"dysel_variant_fn", "dysel_status"})


def test_header_declares_the_paper_calls():
    names = declared()
    for n in ("dysel_register_variants", "dysel_launch", "dysel_spmv", "dysel_sgemm", "dysel_spmv_prepare",
              "dysel_get_selection", "dysel_spmv_sharded", "dysel_sgemm_sharded"):
        assert n in names


def test_library_builds_and_exports_every_symbol():
    from paper_conf_asplos_changkh16_b200 import build
    lib = build.build()
    L = ctypes.CDLL(lib)
    missing = [n for n in declared() if not hasattr(L, n)]
    assert not missing, missing


def test_binding_loads_and_names_match():
    from paper_conf_asplos_changkh16_b200 import dysel
    for n in declared():
        assert hasattr(dysel, n), n


def test_status_strings_and_partition_cpu():
    from paper_conf_asplos_changkh16_b200 import dysel
    assert dysel.dysel_status_str(0) == b"DYSEL_OK"
    assert dysel.dysel_status_str(2) == b"DYSEL_ERR_UNSUPPORTED"
    import numpy as np
    from oracle import partition
    from workloads import d4_powerlaw
    A = d4_powerlaw(n=50_000, lmax=2000)
    for world in (1, 2, 3, 4, 8):
        assert dysel.partition_rows(A.row_ptr, world) == partition.partition_rows(A.row_ptr, world)
    # degenerate: empty matrix, world > rows
    rp = np.zeros(1, np.int32)
    assert dysel.partition_rows(rp, 4) == [0, 0, 0, 0, 0]


def test_sm100a_sass_has_tcgen05():
    import shutil
    import subprocess
    from paper_conf_asplos_changkh16_b200 import build
    lib = build.build()
    if not shutil.which("cuobjdump"):
        pytest.skip("cuobjdump not found")
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    assert "UTCHMMA" in out and "LDTM" in out     # tcgen05.mma / tcgen05.ld
    assert "sm_100a" in subprocess.run(["cuobjdump", "-lelf", lib], capture_output=True, text=True).stdout
