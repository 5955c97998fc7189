"""The C-ABI library loads without a GPU, exports every symbol include/kcore.h
declares, and rejects bad arguments before touching the device."""
import ctypes
import os
import re

import pytest

import paper_conf_icde_ahmady0gcz23_b200 as kc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(kcore_[a-z_0-9]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    lib = kc.library()
    names = _declared("kcore.h")
    assert len(names) >= 12
    for name in names:
        assert hasattr(lib, name), name
    assert set(names) == set(kc.EXPORTS)


def test_library_exports_test_hooks():
    lib = kc.library()
    for name in _declared("kcore_test.h"):
        assert hasattr(lib, name), name


def test_generator_library_exports():
    import kcgen
    lib = kcgen._load()
    txt = open(os.path.join(ROOT, "kcgen", "include", "kcgen.h")).read()
    for name in set(re.findall(r"\b(kcg_[a-z_0-9]+)\s*\(", txt)):
        assert hasattr(lib, name), name


def test_strerror_and_version():
    assert kc.strerror(0) == "KCORE_OK"
    for code in (-1, -2, -3, -4, -5, -6):
        assert kc.strerror(code).startswith("KCORE_E")
    assert "sm_100a" in kc.version()


def test_workspace_size_scales_linearly():
    a = kc.kcore_workspace_size(1 << 20, 1 << 24)
    b = kc.kcore_workspace_size(1 << 21, 1 << 24)
    assert 26 * (1 << 20) <= a <= 56 * (1 << 20) + (8 << 20)  # ~52 n B (queues, alive + near lists, bits, degrees) + segment slack
    assert b > a


def test_argument_errors_before_any_launch():
    lib = kc.library()
    dummy = ctypes.c_void_p(0x1000)
    # n < 0, n >= 2^31, m < 0, m >= 2^33, null pointers -> EINVAL without CUDA
    assert lib.kcore_decompose(dummy, dummy, -1, 0, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(dummy, dummy, 1 << 31, 0, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(dummy, dummy, 4, -2, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(dummy, dummy, 4, 1 << 33, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(None, dummy, 4, 2, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(dummy, None, 4, 2, dummy, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(dummy, dummy, 4, 2, None, None) == kc.KCORE_EINVAL
    assert lib.kcore_decompose(None, None, 0, 5, None, None) == kc.KCORE_EINVAL
    # empty graph: OK, no launch
    assert lib.kcore_decompose(None, None, 0, 0, None, None) == kc.KCORE_OK
    assert lib.kcore_decompose_mg_virtual(None, None, -1, 0, 2, None, None, None) in (
        kc.KCORE_EINVAL, kc.KCORE_EUNSUPPORTED)


def test_output_and_mpm_argument_errors_before_any_launch():
    lib = kc.library()
    d = ctypes.c_void_p(0x1000)
    cnt, cnt2 = ctypes.c_int64(7), ctypes.c_int64(7)
    assert lib.kcore_kshell(d, -1, 0, d, ctypes.byref(cnt), None) == kc.KCORE_EINVAL
    assert lib.kcore_kshell(None, 5, 0, d, ctypes.byref(cnt), None) == kc.KCORE_EINVAL
    assert lib.kcore_kshell(None, 0, 3, None, ctypes.byref(cnt), None) == kc.KCORE_OK and cnt.value == 0
    assert lib.kcore_kcore_mask(d, 5, 1, None, None, None) == kc.KCORE_EINVAL
    assert lib.kcore_kcore_mask(d, 1 << 31, 1, d, None, None) == kc.KCORE_EINVAL
    assert lib.kcore_kcore_subgraph(d, d, d, 4, 6, 1, None, ctypes.byref(cnt2), None, None, None,
                                    None) == kc.KCORE_EINVAL
    assert lib.kcore_kcore_subgraph(d, d, d, 4, 6, 1, ctypes.byref(cnt), ctypes.byref(cnt2), d, d, None,
                                    None) == kc.KCORE_EINVAL  # filling needs vmap_out
    assert lib.kcore_kcore_subgraph(None, None, None, 0, 0, 1, ctypes.byref(cnt), ctypes.byref(cnt2), None,
                                    None, None, None) == kc.KCORE_OK
    assert cnt.value == 0 and cnt2.value == 0
    it = ctypes.c_int64(5)
    assert lib.kcore_mpm(d, d, -1, 0, d, -1, ctypes.byref(it), None, None) == kc.KCORE_EINVAL
    assert lib.kcore_mpm(d, None, 4, 6, d, -1, ctypes.byref(it), None, None) == kc.KCORE_EINVAL
    assert lib.kcore_mpm(None, None, 0, 0, None, -1, ctypes.byref(it), None, None) == kc.KCORE_OK
    assert it.value == 0


def test_no_cpu_fallback_in_product_package():
    """The product package never imports the oracle or any CPU decomposition."""
    pkg = os.path.join(ROOT, "paper_conf_icde_ahmady0gcz23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "networkx" not in src, f


def test_committed_traffic_capture_matches_kernel_code():
    """profiles/ncu_traffic_C4.json (bench.py's roofline.traffic) was captured on
    exactly the k_persistent code this tree builds (sha256 of its SASS)."""
    import json
    import shutil
    import bench
    if shutil.which("cuobjdump") is None:
        pytest.skip("cuobjdump not available")
    sha = bench._lib_sha()
    assert sha and len(sha) == 64
    tj = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic_C4.json")))
    assert tj["sass_sha256"] == sha
    assert tj["dram_bytes_per_launch"] > 0 and tj["dram_bytes_per_launch_window_off"] > 0
