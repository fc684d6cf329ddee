"""CPU-side checks of the boundary: the library builds, loads and exports every
symbol include/etg.h declares; the binding refuses to run without a GPU (no
CPU fallback); host-side size logic."""
import ctypes
import os
import re

import pytest
import torch

import paper_conf_ipps_wangzlg19_b200 as etg
from paper_conf_ipps_wangzlg19_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    _build.build()
    return etg.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "etg.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(etg_[a-z0-9_]+)\s*\(", src)
    return sorted(set(names))


def test_header_declares_the_boundary():
    names = declared_functions()
    for required in ("etg_load_csr", "etg_bfs", "etg_sssp", "etg_cc", "etg_free",
                     "etg_workspace_bytes", "etg_udc_slices", "etg_run_host"):
        assert required in names


def test_library_exports_every_declared_symbol(L):
    raw = ctypes.CDLL(_build.LIB)
    for name in declared_functions():
        assert hasattr(raw, name), f"libetg.so does not export {name}"


def test_sm100a_code_in_library(L):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _build.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings(L):
    assert L.etg_status_str(0) == b"ETG_OK"
    assert L.etg_status_str(-7) == b"ETG_ENOWEIGHTS"


def test_workspace_bytes_monotone(L):
    o = etg.Options(32, 0)
    a = L.etg_workspace_bytes(1000, 10_000, ctypes.byref(o))
    b = L.etg_workspace_bytes(2000, 10_000, ctypes.byref(o))
    c = L.etg_workspace_bytes(2000, 1_000_000, ctypes.byref(etg.Options(1, 0)))
    assert 0 < a < b < c
    # C2-sized workspace stays small next to the CSR (8 n B of col/w per edge x 16):
    # snap, F, B, D, S, Lx, Lfull (7 arrays of n words) + the bitmaps Q, V + tile_first + scan descriptors
    n, m = 1 << 22, 67_000_000
    ws = L.etg_workspace_bytes(n, m, ctypes.byref(o))
    assert 28 * n < ws < 30 * n


def test_load_rejects_bad_arguments_without_gpu(L):
    h = ctypes.c_void_p()
    o = etg.Options(32, 0)
    rc = L.etg_load_csr(ctypes.byref(h), 10, 5, None, None, None, None, 0, None, ctypes.byref(o), None, 0, 0)
    assert rc == -1  # ETG_EINVAL before touching the device
    rc = L.etg_load_csr(ctypes.byref(h), 1 << 33, 5, ctypes.c_void_p(256), ctypes.c_void_p(256),
                        None, ctypes.c_void_p(256), 1 << 40, None, ctypes.byref(o), None, 0, 0)
    assert rc == -6  # ETG_ERANGE: n > 2^32 - 2
    rc = L.etg_load_csr(ctypes.byref(h), 10, 1 << 32, ctypes.c_void_p(256), ctypes.c_void_p(256),
                        None, ctypes.c_void_p(256), 1 << 40, None, ctypes.byref(o), None, 0, 0)
    assert rc == -6  # m >= 2^32 needs u64 offsets
    push = etg.Options(32, etg.PUSH)
    rc = L.etg_load_csr(ctypes.byref(h), 10, 5, ctypes.c_void_p(256), ctypes.c_void_p(256),
                        None, ctypes.c_void_p(256), 1 << 40, None, ctypes.byref(push), None, 0, 10)
    assert rc == -1  # ETG_PUSH needs a communicator


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback():
    off = torch.zeros(2, dtype=torch.int32)
    col = torch.zeros(0, dtype=torch.int32)
    with pytest.raises(etg.EtgError):
        etg.Graph(off, col)


def test_u32_bit_packing():
    x = torch.tensor([0, 1, 2**31 - 1, 2**31, 2**32 - 1], dtype=torch.int64)
    y = etg._as_u32_bits(x)
    assert y.dtype == torch.int32
    assert etg.to_u32_numpy(y).tolist() == [0, 1, 2**31 - 1, 2**31, 2**32 - 1]
