"""C-ABI library checks that need no GPU: libvbatched.so loads, exports every symbol that
include/vbatched.h declares, and host-scalar argument checks return -p before any CUDA work."""
import os
import re

import numpy as np

import paper_conf_ipps_abdelfattahhtd16_b200 as vb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    hdr = open(os.path.join(ROOT, "include", "vbatched.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(vbatched_\w+)\s*\(", hdr)))


def test_header_symbols_exported():
    lib = vb.lib()
    syms = _declared_symbols()
    assert len(syms) >= 14, syms
    for s in syms:
        assert hasattr(lib, s), f"{s} declared in include/vbatched.h but not exported"


def test_python_binding_names_match_header():
    for s in _declared_symbols():
        assert hasattr(vb, s), f"binding lacks {s}"


def test_version_string():
    v = vb.vbatched_version()
    assert "sm_100a" in v and "DMMA" in v


def test_host_argument_checks_without_gpu():
    # host scalars are checked before any CUDA call (include/vbatched.h conventions)
    assert vb.vbatched_dpotrf("X", 0, 0, 0, 0, 1, 4, stream=0, check=False) == -1
    assert vb.vbatched_dpotrf("u", 0, 0, 0, 0, -1, 4, stream=0, check=False) == -6  # 'U' accepted
    assert vb.vbatched_dpotrf("U", 0, 0, 0, 0, 0, 4, stream=0, check=False) == 0
    assert vb.vbatched_dpotrf("L", 0, 0, 0, 0, -1, 4, stream=0, check=False) == -6
    assert vb.vbatched_dpotrf("L", 0, 0, 0, 0, 1, -3, stream=0, check=False) == -7
    assert vb.vbatched_dpotrf("L", 0, 0, 0, 0, 0, 0, stream=0, check=False) == 0
    assert vb.vbatched_dpotrf_nomax("L", 0, 0, 0, 0, -2, stream=0, check=False) == -6
    assert vb.vbatched_dgemm("Q", "N", 0, 0, 0, 1, 0, 0, 0, 0, 0, 0, 0, 1, 1, 1, 1, stream=0,
                             check=False) == -1
    assert vb.vbatched_dsyrk("L", "X", 0, 0, 1, 0, 0, 0, 0, 0, 1, 1, 1, stream=0, check=False) == -2
    assert vb.vbatched_dtrsm("R", "L", "T", "Z", 0, 0, 1, 0, 0, 0, 0, 1, 1, 1, stream=0,
                             check=False) == -4
    assert vb.vbatched_dpotrf_scan("L", 0, 0, 0, 5, 4, 0, stream=0, check=False) == -7
    assert vb.vbatched_dpotrf_factor("L", 0, 0, 0, 0, 5, 4, 0, stream=0, check=False) == -8
    assert vb.vbatched_dpotrf_workspace_size(1000) >= 4000


def test_host_api_argument_checks_and_codes():
    n = np.array([3, -1, 5, 8], dtype=np.int32)
    ld = np.array([3, 4, 4, 8], dtype=np.int32)
    info = np.zeros(4, dtype=np.int32)
    ptrs = np.zeros(4, dtype=np.int64)
    assert vb.vbatched_dpotrf_host("L", n, ptrs, ld, info, 4, -1, check=False) == -7
    assert vb.vbatched_dpotrf_host("Q", n, ptrs, ld, info, 4, 8, check=False) == -1


def test_kernel_launch_count():
    assert vb.vbatched_dpotrf_kernel_launches(0) == 0
    assert vb.vbatched_dpotrf_kernel_launches(32) == 1
    assert vb.vbatched_dpotrf_kernel_launches(100) >= 3
