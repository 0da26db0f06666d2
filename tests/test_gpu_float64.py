"""GPU parity in float64, the paper's own precision ("double (64-bit)
numbers"), through the C ABI.

Two input recipes (sat_inputs):
  * "unit"   k * 2^-24 in [0, 1): every partial sum below 2^29 is exact, so
    every variant, tile shape and look-back order must equal the float64
    oracle BIT FOR BIT (sizes up to ~23K^2);
  * "unit53" full 53-bit mantissas: rounding depends on the summation order.
    Each b[i][j] is a sum of positive terms whose addition tree (row scans,
    chunk carries, column prefix, add vectors, look-back aggregates) is at
    most i + j + 128 deep, so |g - o| <= 2 (i + j + 128) u o elementwise
    (u = 2^-53; the factor 2 covers the oracle's own rounding).  4R1W
    subtracts (Formula (1)), so it gets the SAT(delta) bound of DESIGN.md R16.
"""
import numpy as np
import pytest
import torch

import oracle
from sat_inputs import make_np, make_torch

pytestmark = pytest.mark.gpu

VARIANTS = ["1r1w", "2r2w", "2r1w", "1+rr1w", "4r4w", "4r1w"]
U = 2.0 ** -53


@pytest.fixture(scope="module")
def libsat():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_kasagini14_b200 as m
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def exact(got, ref):
    got = got.cpu().numpy() if isinstance(got, torch.Tensor) else got
    if not np.array_equal(got, ref):
        bad = np.argwhere(got != ref)
        raise AssertionError(f"{len(bad)} mismatches, first at {bad[:5].tolist()}")


def within_order_bound(got, ref, variant):
    got = got.cpu().numpy() if isinstance(got, torch.Tensor) else got
    n, m = ref.shape
    err = np.abs(got - ref)
    if variant == "4r1w":
        bound = 3 * U * np.cumsum(np.cumsum(2 * ref + 1, axis=0), axis=1) * 1.01
    else:
        depth = np.arange(n)[:, None] + np.arange(m)[None, :] + 128
        bound = 2 * depth * U * ref
    assert (err <= bound).all(), f"max err/bound {(err / np.maximum(bound, 1e-300)).max()}"


@pytest.mark.parametrize("variant", VARIANTS)
def test_fig3_float64(libsat, fig3, variant):
    a, _, b = fig3
    y = libsat.sat(dev(a.astype(np.float64)), variant=variant)
    assert y.dtype == torch.float64
    exact(y, b.astype(np.float64))


SHAPES = [(1, 1), (1, 5), (5, 1), (3, 5), (15, 127), (16, 128), (17, 129), (63, 255),
          (64, 256), (65, 257), (127, 129), (200, 1000), (1080, 1920), (333, 1001), (2049, 513)]


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: f"{s[0]}x{s[1]}")
def test_shapes_float64(libsat, variant, shape):
    a = make_np(*shape, "float64", "unit", seed=shape[0] * 5 + shape[1])
    exact(libsat.sat(dev(a), variant=variant), oracle.sat(a))
    a53 = make_np(*shape, "float64", "unit53", seed=shape[1])
    within_order_bound(libsat.sat(dev(a53), variant=variant), oracle.sat(a53), variant)


@pytest.mark.parametrize("tile_rows", [16, 32, 64, 128])
@pytest.mark.parametrize("generic", [False, True])
@pytest.mark.parametrize("variant", ["1r1w", "2r2w", "2r1w", "1+rr1w"])
def test_tile_configs_float64(libsat, tile_rows, generic, variant):
    a = make_np(700, 1300, "float64", "unit", seed=tile_rows)
    exact(libsat.sat(dev(a), variant=variant, tile_rows=tile_rows, force_generic=generic),
          oracle.sat(a))
    if not generic and (variant == "1r1w" or (variant in ("2r1w", "1+rr1w") and tile_rows <= 64)):
        assert libsat.last_tile_rows() == tile_rows


def test_float64_inplace_batched_jitter(libsat):
    a = make_np(129, 700, "float64", "unit", seed=9, batch=3)
    got = libsat.sat_batched(dev(a)).cpu().numpy()
    for i in range(3):
        exact(got[i], oracle.sat(a[i]))
    b = make_np(1000, 1024, "float64", "unit", seed=10)
    x = dev(b)
    ref = oracle.sat(b)
    for th in (16, 32, 64):
        exact(libsat.sat(x, tile_rows=th, jitter=20000), ref)
    y = libsat.sat(x, out=x)
    assert y.data_ptr() == x.data_ptr()
    exact(x, ref)


@pytest.mark.parametrize("nseg", [2, 5])
def test_float64_segments(libsat, nseg):
    a = make_np(64 * 40 + 7, 2048, "float64", "unit", seed=nseg)
    exact(libsat.sat(dev(a), tile_rows=32, segments=nseg), oracle.sat(a))


def test_float64_seeded_sharded_totals(libsat):
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    full = make_np(900, 1100, "float64", "unit", seed=8)
    ref = oracle.sat(full)
    r0 = 311
    strip = dev(full[r0:])
    exact(libsat.sat_seeded(strip, carry_row=dev(oracle.column_totals(full[:r0]))), ref[r0:])
    exact(libsat.sat_seeded(strip, sat_row=dev(ref[r0 - 1])), ref[r0:])
    exact(libsat.column_totals(dev(full)), oracle.column_totals(full))
    P = 3
    bounds = [partition_rows(900, P, p) for p in range(P)]
    strips = [dev(full[a:b]) for a, b in bounds]
    totals = [libsat.column_totals(s) for s in strips]
    totals[-1] = torch.zeros_like(totals[-1])
    outs = []
    for p in range(P):
        def ag(send, recv, p=p):
            torch.cuda.synchronize()
            recv.copy_(torch.stack(totals))
        o, st = libsat.sat_sharded_abi(strips[p], p, P, ag)
        outs.append(o.cpu().numpy())
        assert st["allgather_bytes"] == P * 1100 * 8
    exact(np.concatenate(outs), ref)


@pytest.mark.parametrize("pinned", [True, False])
def test_float64_host_end_to_end(libsat, pinned):
    a = make_np(3000, 2048, "float64", "unit", seed=12)
    x = torch.from_numpy(a)
    if pinned:
        x = x.pin_memory()
    exact(libsat.sat_host(x).numpy(), oracle.sat(a))


@pytest.mark.slow
def test_float64_16k_full(libsat):
    """16384^2 float64 in the bench launch configuration: bit-exact (dyadic)."""
    n = 16384
    x = make_torch(n, n, "float64", "unit", seed=3003, device="cuda")
    y = libsat.sat(x).cpu().numpy()
    a = x.cpu().numpy()
    st = oracle.Stream(n, False)
    for r0 in range(0, n, 1024):
        exact(y[r0:r0 + 1024], st.feed(a[r0:r0 + 1024]))


@pytest.mark.parametrize("shape", [(1000, 1100), (128 * 100 + 7, 700), (300, 64 * 33 + 4), (129, 4)],
                         ids=lambda s: f"{s[0]}x{s[1]}")
def test_float64_th128_narrow_chunks(libsat, shape):
    """float64 at TH 128 runs 64-column chunks (two doubles per lane, the int32
    TH-128 geometry): partial last chunks, many bands, segments, seeds, jitter."""
    a = make_np(*shape, "float64", "unit", seed=shape[0] % 97)
    ref = oracle.sat(a)
    x = dev(a)
    exact(libsat.sat(x, tile_rows=128), ref)
    assert libsat.last_tile_rows() == 128
    exact(libsat.sat(x, tile_rows=128, segments=3), ref)
    exact(libsat.sat(x, tile_rows=128, jitter=20000), ref)
    if shape[0] > 300:
        r0 = 257
        exact(libsat.sat_seeded(dev(a[r0:]), carry_row=dev(oracle.column_totals(a[:r0]))), ref[r0:])
    b = make_np(*shape, "float64", "unit", seed=3, batch=2)
    got = libsat.sat_batched(dev(b), tile_rows=128).cpu().numpy()
    for i in range(2):
        exact(got[i], oracle.sat(b[i]))
