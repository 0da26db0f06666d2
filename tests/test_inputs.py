"""The shared input generator: numpy and torch twins agree bit for bit, strips
and batches reproduce the full tensor, value ranges are as documented."""
import numpy as np
import pytest
import torch

from sat_inputs import make_np, make_torch


@pytest.mark.parametrize("dtype,dist", [("int32", "u32"), ("int32", "u8"), ("int32", "ones"),
                                        ("float32", "unit"), ("float32", "ones"),
                                        ("float64", "unit"), ("float64", "unit53"),
                                        ("float64", "ones")])
def test_numpy_torch_twins(dtype, dist):
    a = make_np(37, 53, dtype, dist, seed=123)
    t = make_torch(37, 53, dtype, dist, seed=123, chunk_rows=5).numpy()
    assert a.dtype == t.dtype and np.array_equal(a.view(np.uint32), t.view(np.uint32))


def test_strip_and_batch_consistency():
    full = make_np(40, 33, "int32", "u32", seed=5)
    assert np.array_equal(make_np(15, 33, "int32", "u32", seed=5, row0=10), full[10:25])
    assert np.array_equal(make_torch(15, 33, "int32", "u32", seed=5, row0=10).numpy(), full[10:25])
    bt = make_np(4, 10, "float32", "unit", seed=3, batch=3)
    flat = make_np(12, 10, "float32", "unit", seed=3)
    assert np.array_equal(bt.reshape(12, 10), flat)
    assert np.array_equal(make_torch(4, 10, "float32", "unit", seed=3, batch=3).numpy(), bt)


def test_ranges():
    f = make_np(64, 64, "float32", "unit", seed=1)
    assert f.min() >= 0.0 and f.max() < 1.0
    assert np.array_equal(np.floor(f.astype(np.float64) * 2**24), f.astype(np.float64) * 2**24)
    u8 = make_np(64, 64, "int32", "u8", seed=1)
    assert u8.min() >= 0 and u8.max() <= 255
    u = make_np(64, 64, "int32", "u32", seed=1)
    assert u.min() < -2**30 and u.max() > 2**30
    assert not np.array_equal(make_np(8, 8, seed=1), make_np(8, 8, seed=2))


def test_float64_ranges():
    d = make_np(64, 64, "float64", "unit", seed=1)
    assert np.array_equal(d, make_np(64, 64, "float32", "unit", seed=1).astype(np.float64))
    e = make_np(64, 64, "float64", "unit53", seed=1)
    assert e.min() >= 0.0 and e.max() < 1.0
    assert np.array_equal(np.floor(e * 2**53), e * 2**53)
    assert (np.floor(e * 2**24) != e * 2**24).any()       # genuinely finer than 2^-24
