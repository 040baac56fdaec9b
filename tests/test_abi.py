"""C-ABI boundary checks that need no GPU: the library loads, exports every
symbol include/stf_cholesky.h declares, and validates arguments LAPACK-style
before touching any device."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_sc_augonnetasg24_b200 as stf
from paper_conf_sc_augonnetasg24_b200 import _abi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "stf_cholesky.h")
HARNESS = os.path.join(ROOT, "include", "stf_harness.h")


def header_functions(path=HEADER):
    src = open(path).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(stf_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_planned_boundary():
    fns = header_functions()
    for f in ("stf_cholesky_init", "stf_potrf", "stf_finalize", "stf_last_error"):
        assert f in fns


def test_library_exports_every_declared_symbol():
    out = subprocess.run(["nm", "-D", "--defined-only", _abi.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (stf_[a-z_0-9]+)", out))
    missing = [f for f in header_functions() + header_functions(HARNESS) if f not in exported]
    assert not missing, missing
    assert sorted(_abi.EXPORTS) == header_functions()
    assert sorted(_abi.HARNESS_EXPORTS) == header_functions(HARNESS)
    assert not set(_abi.EXPORTS) & set(_abi.HARNESS_EXPORTS)


def test_library_has_sm100a_code():
    out = subprocess.run(["cuobjdump", "--list-elf", _abi.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _desc_host(ptr=None, ld=4):
    return _abi.stf_matrix_desc(stf.STF_DESC_HOST_COLMAJOR, 0, ld, ptr, 0, 0, None)


@pytest.mark.parametrize(
    "n,nb,uplo,code",
    [(-1, 2, b"L", -1), (4, 0, b"L", -2), (4, 3, b"L", -2), (6, 4, b"L", -2), (4, 2, b"X", -3)],
)
def test_argument_validation_without_gpu(n, nb, uplo, code):
    buf = (ctypes.c_double * 64)()
    d = _desc_host(ctypes.cast(buf, ctypes.c_void_p), ld=8)
    assert _abi.stf_potrf(n, nb, uplo, ctypes.byref(d), 1) == code
    assert len(_abi.stf_last_error()) > 0


def test_bad_descriptor_codes():
    assert _abi.stf_potrf(4, 2, b"L", None, 1) == -4
    buf = (ctypes.c_double * 64)()
    d = _desc_host(ctypes.cast(buf, ctypes.c_void_p), ld=2)  # ld < n
    assert _abi.stf_potrf(4, 2, b"L", ctypes.byref(d), 1) == -4
    d = _abi.stf_matrix_desc(7, 0, 4, None, 0, 0, None)
    assert _abi.stf_potrf(4, 2, b"L", ctypes.byref(d), 1) == -4
    # TILED requires uplo L and p*q == ngpus
    d = _abi.stf_matrix_desc(stf.STF_DESC_TILED_2DBC, 0, 0, None, 1, 2, None)
    assert _abi.stf_potrf(4, 2, b"U", ctypes.byref(d), 2) == -3
    assert _abi.stf_potrf(4, 2, b"L", ctypes.byref(d), 1) == -4


def test_not_initialised_and_n_zero_order():
    buf = (ctypes.c_double * 64)()
    d = _desc_host(ctypes.cast(buf, ctypes.c_void_p), ld=8)
    assert _abi.stf_potrf(4, 2, b"L", ctypes.byref(d), 0) == -5
    assert _abi.stf_finalize() == -100


def test_init_without_gpu_fails_cleanly():
    from conftest import gpu_available
    if gpu_available():
        pytest.skip("GPU present")
    assert _abi.stf_cholesky_init(1, None) == -101
    assert b"CUDA" in _abi.stf_last_error() or b"device" in _abi.stf_last_error()


OPTIONS = {"graph": (1, 0), "dataflow": (1, 0), "trsm": (3, 1), "streams": (32, 3), "serial": (0, 1),
           "priority": (1, 0), "grid_p": (0, 2), "lookahead": (1, 0), "threads": (8, 2), "trsm_split": (4, 2), "push": (0, 2),
           "trsm_res_tail": (-1, 0), "trsm_rows": (128, 64), "trsm_res_split": (2, 1), "stream_pool": (0, 1),
           "order_mode": (-1, 2), "order_tail": (-1, 0), "order_asap": (0, 1), "sched_width": (0, 3), "prio_mode": (0, 2),
           "ooc_reorder": (1, 0), "dev_order": (0, 1), "ooc_budget_pct": (-1, 40), "host_stream_budget_pct": (90, 75),
           "host_eager": (0, 1), "mem_cap_tiles": (0, 10), "ooc_order": (-1, 0), "host_stream": (1, 0), "pdl": (1, 0), "pdl_lead": (-1, 16), "potrf_split": (1, 0), "potrf_ctas": (0, 24),
           "debug_skip": (0, 8), "debug_trace": (0, 1), "nvtx": (0, 1), "gemm_merge": (2, 0), "gemm_group": (-1, 4)}


@pytest.mark.parametrize("name,value", [("trsm_rows", 48), ("mem_cap_tiles", 2), ("push", 3), ("order_mode", 1),
                                        ("stream_pool", 3), ("ooc_budget_pct", 5), ("streams", 0)])
def test_options_reject_out_of_range(name, value):
    before = stf.get_option(name)
    with pytest.raises(stf.StfError):
        stf.set_option(name, value)
    assert stf.get_option(name) == before


def test_environment_options_are_validated_at_init(tmp_path):
    """An out-of-range STF_<NAME> is rejected at stf_cholesky_init (-105) before any
    device work (in a GPU-less process the device probe fails first: -101)."""
    import subprocess
    import sys
    code = ("import ctypes, sys; sys.path.insert(0, %r); from paper_conf_sc_augonnetasg24_b200 import _abi; "
            "print(_abi.stf_cholesky_init(1, None))" % ROOT)
    env = dict(os.environ, STF_MEM_CAP_TILES="2")
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, timeout=120)
    assert r.stdout.strip() in ("-105", "-101"), r.stdout + r.stderr


def test_options_roundtrip_without_gpu():
    # every option the header documents can be set and read back
    hdr = open(HEADER).read()
    for name, (dflt, other) in OPTIONS.items():
        assert '"%s"' % name in hdr, name
        stf.set_option(name, other)
        assert stf.get_option(name) == other
        stf.set_option(name, dflt)
        assert stf.get_option(name) == dflt
    with pytest.raises(stf.StfError):
        stf.set_option("nonsense", 1)
