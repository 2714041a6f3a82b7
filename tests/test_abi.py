"""C-ABI checks that need no GPU: the library loads, exports every symbol include/memxct.h
declares, validates arguments, enforces plan state, and refuses to run without a CUDA device
(there is no CPU fallback)."""
import ctypes
import os
import re

import pytest

from conftest import ROOT

pytestmark = pytest.mark.filterwarnings("ignore")


@pytest.fixture(scope="module")
def L():
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext, memxct
    build_ext.build()
    return memxct.lib()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "memxct.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(memxct_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    from paper_conf_sc_hidayetoglubgrg19_b200 import memxct
    decl = declared_symbols()
    assert len(decl) >= 20
    assert sorted(memxct.SYMBOLS) == decl
    for name in decl:
        assert hasattr(L, name), name


def test_binary_is_sm100a(L):
    import subprocess
    from paper_conf_sc_hidayetoglubgrg19_b200 import memxct
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", memxct.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _plan(L, n=8, m=4, c=8):
    h = ctypes.c_void_p()
    assert L.memxct_plan_create(n, m, c, ctypes.byref(h)) == 0
    return h


def test_create_validates_sizes(L):
    h = ctypes.c_void_p()
    assert L.memxct_plan_create(0, 4, 4, ctypes.byref(h)) == 1
    assert L.memxct_plan_create(8, -1, 4, ctypes.byref(h)) == 1
    assert L.memxct_plan_create(65536, 4, 4, ctypes.byref(h)) == 1   # n*n >= 2^31
    assert b"n" in L.memxct_last_error()
    assert L.memxct_plan_create(8, 4, 4, None) == 1


def test_options_validated_and_readable(L):
    h = _plan(L)
    assert L.memxct_plan_set_option(h, 3, 70000) == 1          # BUFFER_ENTRIES > 49152
    assert L.memxct_plan_set_option(h, 2, 48) == 1             # PART_ROWS not a multiple of 32
    assert L.memxct_plan_set_option(h, 0, 12) == 1             # tile not a power of two
    assert L.memxct_plan_set_option(h, 99, 1) == 1             # unknown option
    assert L.memxct_plan_set_option(h, 2, 256) == 0
    v = ctypes.c_int64()
    assert L.memxct_plan_get_option(h, 2, ctypes.byref(v)) == 0 and v.value == 256
    assert L.memxct_plan_destroy(h) == 0
    assert L.memxct_plan_destroy(None) == 0                    # NULL-safe


def test_state_errors_before_build(L):
    h = _plan(L)
    z = ctypes.c_void_p(1)
    assert L.memxct_forward(h, z, z, None) == 2
    assert L.memxct_back(h, z, z, None) == 2
    assert L.memxct_cg(h, z, z, 3, None, None) == 2
    cnt = ctypes.c_int64()
    assert L.memxct_local_size(h, 0, ctypes.byref(cnt)) == 2
    assert L.memxct_plan_set_comm(h, 2, 2, None, 0) == 1        # rank out of range
    L.memxct_plan_destroy(h)


def test_status_strings(L):
    assert L.memxct_status_string(0) == b"MEMXCT_OK"
    assert L.memxct_status_string(4) == b"MEMXCT_ERR_CUDA"


def test_no_cpu_fallback_without_gpu(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    h = _plan(L)
    assert L.memxct_build(h, None) == 4                        # MEMXCT_ERR_CUDA: no device
    assert b"no CPU fallback" in L.memxct_last_error() or b"CUDA" in L.memxct_last_error()
    L.memxct_plan_destroy(h)


def test_read_ceiling_validates_arguments(L):
    g = ctypes.c_double()
    assert L.memxct_read_ceiling(8, 1, ctypes.byref(g), None) == 1     # < 16 bytes
    assert L.memxct_read_ceiling(1 << 20, 0, ctypes.byref(g), None) == 1  # reps < 1
    assert L.memxct_read_ceiling(1 << 20, 1, None, None) == 1          # NULL output
