"""GPU parity of the hierarchical look-back: groups of
hg bands publish group sums, so a walk visits its own group band by band and
then one word per group above.  Results must be identical to the flat walk
(int32 bit-exact, float32 within 1e-5 of the float64 oracle) for every group
size, band height, segment split, batch and dtype, under publication jitter,
including group sizes that do not divide the band count and groups larger
than the band count (flat)."""
import numpy as np
import pytest
import torch

import oracle
from sat_inputs import make_np

pytestmark = pytest.mark.gpu
FTOL = 1e-5


@pytest.fixture(scope="module")
def libsat():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_kasagini14_b200 as m
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def gen(n, m, dtype, seed=1):
    return make_np(n, m, dtype, "u32" if dtype == "int32" else "unit", seed=seed)


def check(got, ref, dtype):
    got = got.cpu().numpy() if isinstance(got, torch.Tensor) else got
    if dtype == "int32":
        if not np.array_equal(got, ref):
            bad = np.argwhere(got != ref)
            raise AssertionError(f"{len(bad)} mismatches, first at {bad[:5].tolist()}")
    else:
        err = oracle.max_rel_err(got, ref)
        assert err <= FTOL, f"max rel err {err}"


@pytest.mark.parametrize("hg", [-1, 2, 3, 4, 8, 16, 1000])
@pytest.mark.parametrize("tile_rows", [16, 32, 64, 128])
def test_group_sizes(libsat, hg, tile_rows):
    for dtype in ("int32", "float32"):
        for shape in [(3000, 2500), (tile_rows * 37 + 5, 777 * 4)]:
            a = gen(*shape, dtype, seed=hg % 97 + tile_rows)
            check(libsat.sat(dev(a), tile_rows=tile_rows, lookback_group=hg), oracle.sat(a), dtype)


@pytest.mark.parametrize("hg", [2, 5, 8])
def test_jitter(libsat, hg):
    """Random publication delays shuffle which words a walk meets (aggregate,
    inclusive, group aggregate, group inclusive, not yet published)."""
    for th in (32, 64, 128):
        a = gen(4000, 2600, "int32", seed=th + hg)
        ref = oracle.sat(a)
        x = dev(a)
        for _ in range(2):
            check(libsat.sat(x, tile_rows=th, jitter=20000, lookback_group=hg), ref, "int32")
        af = gen(4000, 1300, "float32", seed=th)
        check(libsat.sat(dev(af), tile_rows=th, jitter=20000, lookback_group=hg), oracle.sat(af), "float32")


@pytest.mark.parametrize("nseg", [2, 5])
@pytest.mark.parametrize("hg", [4, 8])
def test_segments_and_batch(libsat, nseg, hg):
    kw = dict(tile_rows=128, segments=nseg, lookback_group=hg)
    a = gen(20000, 3000, "int32", seed=nseg + hg)
    ref = oracle.sat(a)
    x = dev(a)
    check(libsat.sat(x, **kw), ref, "int32")
    check(libsat.sat(x, jitter=20000, **kw), ref, "int32")
    b = gen(3 * 1100, 1920, "int32", seed=hg).reshape(3, 1100, 1920)
    got = libsat.sat_batched(dev(b), tile_rows=32, lookback_group=hg, segments=nseg).cpu().numpy()
    for i in range(3):
        assert np.array_equal(got[i], oracle.sat(b[i])), i


@pytest.mark.parametrize("hg", [3, 8])
def test_float64_and_2r2w(libsat, hg):
    a = gen(5000, 1500, "float64", seed=hg)
    for th in (32, 64, 128):
        y = libsat.sat(dev(a), tile_rows=th, lookback_group=hg)
        check(y, oracle.sat(a), "float64")
    ai = gen(3000, 2000, "int32", seed=hg)
    check(libsat.sat(dev(ai), variant="2r2w", lookback_group=hg), oracle.sat(ai), "int32")


def test_repeated_calls_group_tags(libsat):
    """Group words are never cleared between calls either: per-launch tags
    keep the previous call's group sums from being taken."""
    for k in range(12):
        shape = (2000 + 131 * k, 300 + 97 * k)
        a = gen(*shape, "int32", seed=200 + k)
        check(libsat.sat(dev(a), tile_rows=32, lookback_group=4 + k % 5), oracle.sat(a), "int32")


def test_bad_group_rejected(libsat):
    x = dev(gen(64, 64, "int32"))
    for bad in (1, -2):
        with pytest.raises(Exception):
            libsat.sat(x, lookback_group=bad)


def test_automatic_choice(libsat):
    """Groups of 4 for one-wave launches of bands <= 64 rows, flat at TH 128
    and for many waves."""
    for shape, dtype, want in [((4096, 4096), "float32", 4), ((6144, 6144), "int32", 4),
                               ((16384, 2048), "int32", 0), ((20480, 1024), "int32", 0),
                               ((60, 300), "int32", 0), ((100, 300), "int32", 4)]:
        a = gen(*shape, dtype, seed=shape[0])
        check(libsat.sat(dev(a)), oracle.sat(a), dtype)
        assert libsat.last_lookback_group() == want, (shape, libsat.last_tile_rows(), libsat.last_lookback_group())
    a = gen(3000, 2000, "int32", seed=9)
    check(libsat.sat(dev(a), lookback_group=-1), oracle.sat(a), "int32")
    assert libsat.last_lookback_group() == 0


def test_group_words_across_tag_resets(libsat):
    """With a tiny tag space the descriptors (group words included: they live
    in the same buffer) are cleared whenever the tags run out; group words of
    earlier calls must never be taken for this call's."""
    libsat.set_tag_space(300000)
    try:
        for k in range(30):
            shape = (1500 + 61 * k, 700 + 13 * k)
            a = gen(*shape, "int32", seed=300 + k)
            check(libsat.sat(dev(a), tile_rows=32, lookback_group=2 + k % 4), oracle.sat(a), "int32")
    finally:
        libsat.set_tag_space(0)


def test_graph_replay_hierarchical(libsat):
    """A captured one-wave launch (automatic groups of 4) replayed on fresh
    inputs, with the device-side ticket base."""
    n, m = 4096, 4096
    x = dev(gen(n, m, "float32", seed=1))
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        y = libsat.sat(x)
    s.synchronize()
    assert libsat.last_lookback_group() == 4
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.sat(x, out=y)
    for it in range(3):
        host = gen(n, m, "float32", seed=50 + it)
        x.copy_(dev(host))
        g.replay()
        torch.cuda.synchronize()
        check(y, oracle.sat(host), "float32")
