"""The C-ABI library loads and exports every symbol include/sat.h declares;
host-side validation works without a GPU (no compute calls here)."""
import ctypes
import os
import re

import pytest

import paper_conf_icpp_kasagini14_b200 as libsat

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "sat.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(sat_[a-z0-9_]+)\s*\(", src))
    return sorted(n for n in names if n != "sat_allgather_fn")


def test_every_declared_symbol_is_exported():
    decl = declared_symbols()
    assert len(decl) >= 15
    for name in decl:
        assert hasattr(libsat.lib, name), name
        assert name in libsat.EXPORTED, name


def test_abi_version_and_strings():
    assert libsat.abi_version() == 2
    assert libsat.lib.sat_strerror(0) == b"ok"
    assert libsat.lib.sat_strerror(-1) == b"invalid argument"


L = libsat.lib


def test_validation_without_gpu():
    # bad dtype
    assert L.sat_compute(8, 8, 4, 4, 7, 2, None) == -1
    assert b"dtype" in L.sat_last_error()
    # negative sizes
    assert L.sat_compute(8, 8, -1, 4, 0, 2, None) == -1
    # null pointers with nonzero size
    assert L.sat_compute(None, 64, 4, 4, 0, 2, None) == -1
    # partial overlap
    assert L.sat_compute(4096, 4100, 4, 4, 0, 2, None) == -1
    assert b"overlap" in L.sat_last_error()
    # misaligned
    assert L.sat_compute(4097, 4097 + 1 << 20, 4, 4, 0, 2, None) == -1
    # bad variant (valid pointers, validated before any CUDA call)
    assert L.sat_compute(4096, 1 << 20, 4, 4, 0, 9, None) == -1
    # empty is a no-op, no device needed
    assert L.sat_compute(None, None, 0, 5, 0, 2, None) == 0
    assert L.sat_compute(None, None, 5, 0, 1, 2, None) == 0
    # bad options
    o = libsat.options(tile_rows=40)
    assert L.sat_compute_ex(4096, 1 << 20, 4, 4, 0, 2, ctypes.byref(o), None) == -1
    o = libsat.options(r=1.5)
    assert L.sat_compute_ex(4096, 1 << 20, 4, 4, 0, 3, ctypes.byref(o), None) == -1
    # sharded argument checks
    assert L.sat_compute_sharded(4096, 1 << 20, 4, 4, 0, 2, 2, libsat.ALLGATHER_FN(0),
                                 None, None, None, None) == -1
    assert L.sat_rank_exscan(None, 64, 2, 4, 3, 0, None) == -1
    assert L.sat_sharded_workspace_bytes(1000, 4, 0) == 256 * 16 * 6
    assert L.sat_compute_host(None, None, 0, 3, 0, 2, None) == 0


def test_python_wrapper_rejects_cpu_tensors():
    import torch
    with pytest.raises(ValueError):
        libsat.sat(torch.zeros(4, 4, dtype=torch.int32))
    with pytest.raises(ValueError):
        libsat.sat(torch.zeros(4, 4, 4, dtype=torch.int32))


def test_validation_new_entry_points_without_gpu():
    """float64 / widening / box filter / rectangle sums: argument checks that
    return before any CUDA call."""
    o = libsat.options()
    # widening pairs: only equal, UINT8->INT32, FLOAT32->FLOAT64
    assert L.sat_compute_widening(4096, 3, 1 << 20, 1, 1, 4, 4, ctypes.byref(o), None) == -1
    assert L.sat_compute_widening(4096, 2, 1 << 20, 1, 1, 4, 4, ctypes.byref(o), None) == -1
    assert b"pair" in L.sat_last_error()
    # widening cannot run in place
    assert L.sat_compute_widening(4096, 1, 4096, 2, 1, 4, 4, ctypes.byref(o), None) == -1
    assert b"in place" in L.sat_last_error()
    # float64 alignment and overlap use 8-byte elements
    assert L.sat_compute(4100, 1 << 20, 4, 4, 2, 2, None) == -1
    assert L.sat_compute(4096, 4096 + 64, 4, 4, 2, 2, None) == -1      # 128-B matrices overlap
    assert b"overlap" in L.sat_last_error()
    # box filter: dtype rules, radii, normalize
    assert L.sat_box_filter(4096, 3, 1 << 20, 1, 1, 4, 4, 1, 1, 0, None) == -1   # uint8 -> float
    assert L.sat_box_filter(4096, 1, 1 << 20, 0, 1, 4, 4, 1, 1, 0, None) == -1   # float -> int
    assert L.sat_box_filter(4096, 0, 1 << 20, 0, 1, 4, 4, -1, 1, 0, None) == -1  # radius
    assert L.sat_box_filter(4096, 0, 1 << 20, 0, 1, 4, 4, 1, 1, 1, None) == -1   # normalize int
    assert b"normalize" in L.sat_last_error()
    assert L.sat_box_filter(None, 3, None, 0, 1, 0, 4, 1, 1, 0, None) == 0       # empty
    # rectangle sums
    assert L.sat_rect_sums(None, 0, 1, 4, 4, 64, 3, 128, None) == -1
    assert L.sat_rect_sums(4096, 5, 1, 4, 4, 64, 3, 128, None) == -1
    assert L.sat_rect_sums(None, 0, 1, 4, 4, None, 0, None, None) == 0
    # the 4R4W / 4R1W variant codes are accepted by validation (bad options still fail)
    o = libsat.options(tile_rows=40)
    assert L.sat_compute_ex(4096, 1 << 20, 4, 4, 0, 5, ctypes.byref(o), None) == -1
    assert L.sat_compute_ex(4096, 1 << 20, 4, 4, 0, 6, ctypes.byref(o), None) == -1
    assert b"variant" in L.sat_last_error()


def test_nccl_unique_id_and_argument_checks():
    """In-library NCCL (sat_nccl_*): libnccl.so.2 is dlopen-ed on first use;
    the unique id needs no GPU; bad arguments fail before any NCCL call."""
    a, b = libsat.nccl_unique_id(), libsat.nccl_unique_id()
    assert len(a) == 128 and len(b) == 128 and a != b
    h = ctypes.c_void_p()
    assert L.sat_nccl_comm_create(ctypes.byref(h), a, 2, 2) == -1       # rank >= nranks
    assert L.sat_nccl_comm_create(ctypes.byref(h), None, 0, 1) == -1    # null id
    assert L.sat_nccl_comm_destroy(None) == 0
    stats = libsat.SatShardStats()
    assert L.sat_compute_sharded_nccl(8, 8, 4, 4, 0, 2, None, None, None, ctypes.byref(stats)) == -1
    # sharded variants: 1R1W and 2R2W take the seed; the others are refused
    assert L.sat_compute_sharded_ex(8, 8, 4, 4, 0, 1, 0, 1, libsat.ALLGATHER_FN(0), None, None, None,
                                    None) == -2
