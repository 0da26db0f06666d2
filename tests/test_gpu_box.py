"""GPU parity for the SAT's consumers and widening inputs:
widening 1R1W (uint8 -> int32 sums, float32 -> float64 sums), the box filter
and rectangle-sum queries, through the C ABI, against the
oracle's plain definitions (oracle.sat, oracle.box_filter, oracle.rect_sum).

Integer paths are exact (mod 2^32).  Float32 inputs are dyadic (k 2^-24), so
their float64 SATs and box sums are exact and the float32 box output is the
correctly rounded exact value: compared bit for bit.  Full-mantissa float64
box sums get the SAT-error bound (R17) through four corners.
"""
import numpy as np
import pytest
import torch

import oracle
from sat_inputs import make_np

pytestmark = pytest.mark.gpu
U = 2.0 ** -53


@pytest.fixture(scope="module")
def libsat():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_kasagini14_b200 as m
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def u8img(n, m, seed, batch=None):
    return make_np(n, m, "int32", "u8", seed=seed, batch=batch).astype(np.uint8)


# ------------------------------------------------------------------ widening 1R1W
@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (64, 256), (129, 160), (1080, 1920), (333, 1000),
                                   (2049, 784)], ids=lambda s: f"{s[0]}x{s[1]}")
@pytest.mark.parametrize("generic", [False, True])
def test_widening_uint8(libsat, shape, generic):
    a = u8img(*shape, seed=shape[0])
    y = libsat.sat_widening(dev(a), torch.int32, force_generic=generic)
    assert np.array_equal(y.cpu().numpy(), oracle.sat(a.astype(np.int32)))


@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (64, 256), (129, 160), (1080, 1920), (2049, 784)],
                         ids=lambda s: f"{s[0]}x{s[1]}")
def test_widening_float32_to_float64(libsat, shape):
    a = make_np(*shape, "float32", "unit", seed=shape[1])
    y = libsat.sat_widening(dev(a), torch.float64)
    assert np.array_equal(y.cpu().numpy(), oracle.sat(a))        # exact: dyadic sums in double


def test_widening_batched_tiles_segments(libsat):
    a = u8img(1080, 1920, seed=4, batch=5)
    for th in (64, 128):
        y = libsat.sat_widening(dev(a), torch.int32, tile_rows=th).cpu().numpy()
        for b in range(5):
            assert np.array_equal(y[b], oracle.sat(a[b].astype(np.int32)))
    f = make_np(700, 1300, "float32", "unit", seed=3)
    for th in (16, 32, 64):
        assert np.array_equal(libsat.sat_widening(dev(f), torch.float64, tile_rows=th).cpu().numpy(),
                              oracle.sat(f))
    g = u8img(64 * 40 + 7, 2048, seed=5)
    assert np.array_equal(libsat.sat_widening(dev(g), torch.int32, tile_rows=64, segments=3).cpu().numpy(),
                          oracle.sat(g.astype(np.int32)))


# ------------------------------------------------------------------ box filter
@pytest.mark.parametrize("rr,rc", [(0, 0), (1, 1), (4, 4), (2, 7), (40, 3), (2000, 2000)])
def test_box_uint8_images(libsat, rr, rc):
    a = u8img(270, 480, seed=rr * 31 + rc, batch=3)
    y = libsat.box_filter(dev(a), rr, rc).cpu().numpy()
    assert y.dtype == np.int32
    for b in range(3):
        assert np.array_equal(y[b], oracle.box_filter(a[b].astype(np.int32), rr, rc))


@pytest.mark.parametrize("shape", [(1, 1), (5, 3), (127, 129), (1080, 1920)], ids=lambda s: f"{s[0]}x{s[1]}")
def test_box_int32_wrapping(libsat, shape):
    a = make_np(*shape, "int32", "u32", seed=7)
    assert np.array_equal(libsat.box_filter(dev(a), 3, 5).cpu().numpy(), oracle.box_filter(a, 3, 5))


@pytest.mark.parametrize("normalize", [False, True])
def test_box_float32_exact(libsat, normalize):
    """Dyadic float32 input: float64 SAT and box sums are exact, the float32
    output is the correctly rounded oracle value, bit for bit."""
    a = make_np(540, 960, "float32", "unit", seed=11, batch=2)
    for out_dtype in (torch.float32, torch.float64):
        y = libsat.box_filter(dev(a), 4, 6, normalize=normalize, out_dtype=out_dtype).cpu().numpy()
        for b in range(2):
            ref = oracle.box_filter(a[b], 4, 6, normalize=normalize)
            assert np.array_equal(y[b], ref.astype(y.dtype))


def test_box_float64_full_mantissa(libsat):
    n, m, rr, rc = 300, 500, 3, 9
    a = make_np(n, m, "float64", "unit53", seed=2)
    y = libsat.box_filter(dev(a), rr, rc).cpu().numpy()
    ref = oracle.box_filter(a, rr, rc)
    S = oracle.sat(a)
    i = np.arange(n)[:, None]
    j = np.arange(m)[None, :]
    i1, i2 = np.maximum(0, i - rr), np.minimum(n - 1, i + rr)
    j1, j2 = np.maximum(0, j - rc), np.minimum(m - 1, j + rc)

    def corner(r, c):
        ok = (r >= 0) & (c >= 0)
        rr_, cc_ = np.clip(r, 0, None), np.clip(c, 0, None)
        return np.where(ok, S[rr_, cc_] * (rr_ + cc_ + 128), 0.0), np.where(ok, S[rr_, cc_], 0.0)
    tot_e = np.zeros((n, m))
    tot_m = np.zeros((n, m))
    for r, c in [(i2, j2), (i1 - 1, j2), (i2, j1 - 1), (i1 - 1, j1 - 1)]:
        e, mag = corner(r + 0 * c, c + 0 * r)
        tot_e += e
        tot_m += mag
    bound = 2 * U * tot_e + 4 * U * tot_m + 2 * U * np.abs(ref)
    assert (np.abs(y - ref) <= bound).all()


def test_box_inplace_and_generic(libsat):
    a = make_np(333, 1001, "int32", "u8", seed=9)           # cols % 4 != 0: generic path
    x = dev(a)
    ref = oracle.box_filter(a, 2, 2)
    y = libsat.box_filter(x, 2, 2, out=x)
    assert y.data_ptr() == x.data_ptr()
    assert np.array_equal(x.cpu().numpy(), ref)
    b = u8img(333, 1001, seed=9)
    assert np.array_equal(libsat.box_filter(dev(b), 2, 2).cpu().numpy(), oracle.box_filter(b.astype(np.int32), 2, 2))


# ------------------------------------------------------------------ rectangle queries
def test_rect_sums(libsat):
    rng = np.random.default_rng(0)
    batch, n, m = 3, 300, 400
    a = make_np(n, m, "int32", "u32", seed=13, batch=batch)
    sat = libsat.sat_batched(dev(a))
    K = 5000
    rects = np.stack([rng.integers(-1, batch + 1, K), rng.integers(-20, n + 20, K),
                      rng.integers(-20, m + 20, K), rng.integers(-20, n + 20, K),
                      rng.integers(-20, m + 20, K)], axis=1).astype(np.int32)
    got = libsat.rect_sums(sat, dev(rects)).cpu().numpy()
    refs = [oracle.sat(a[b]) for b in range(batch)]
    for q in range(K):
        b, r0, c0, r1, c1 = rects[q].tolist()
        r0, c0, r1, c1 = max(r0, 0), max(c0, 0), min(r1, n - 1), min(c1, m - 1)
        want = 0
        if 0 <= b < batch and r0 <= r1 and c0 <= c1:
            want = int(np.uint32(oracle.rect_sum(refs[b], r0, c0, r1, c1)).view(np.int32))
        assert int(got[q]) == want, (q, rects[q])
    # float64 SAT of dyadic input: exact rectangle sums equal the input block sums
    f = make_np(200, 300, "float64", "unit", seed=14)
    sf = libsat.sat(dev(f))
    rq = np.array([[0, 10, 20, 150, 250], [0, 0, 0, 199, 299], [0, 5, 5, 5, 5]], dtype=np.int32)
    gf = libsat.rect_sums(sf, dev(rq)).cpu().numpy()
    for q, (_, r0, c0, r1, c1) in enumerate(rq.tolist()):
        assert gf[q] == f[r0:r1 + 1, c0:c1 + 1].sum()


def test_box_filter_cuda_graph(libsat):
    """The box filter (widening 1R1W SAT + box pass) captured in a CUDA graph
    and replayed on fresh uint8 frames (the device-side ticket base,
    DESIGN.md Sec. 4); the workspace is sized by one eager call first."""
    B, n, m, rr, rc = 3, 540, 960, 4, 4
    x = dev(u8img(n, m, seed=1, batch=B))
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        y = libsat.box_filter(x, rr, rc)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.box_filter(x, rr, rc, out=y)
    for it in range(3):
        a = u8img(n, m, seed=50 + it, batch=B)
        x.copy_(dev(a))
        g.replay()
        torch.cuda.synchronize()
        got = y.cpu().numpy()
        for b in range(B):
            assert np.array_equal(got[b], oracle.box_filter(a[b].astype(np.int32), rr, rc)), (it, b)


# ------------------------------------------------------------------ fused box filter (sat_boxf.cuh)
@pytest.mark.parametrize("shape,rr,rc,batch", [
    ((1080, 1920), 4, 4, 3),       # the cfg5-style image batch (r = 4)
    ((1000, 2064), 16, 127, 2),    # largest fused radii; partial last chunk (2064 = 16 x 128 + 16)
    ((50, 16), 3, 9, 4),           # fewer rows than a band, one 16-column chunk
    ((64, 256), 0, 0, 1),          # identity
    ((130, 400), 16, 1, 1),        # window taller than the rows a band owns
    ((777, 1296), 7, 100, 2),
], ids=lambda v: str(v))
def test_box_fused_uint8(libsat, shape, rr, rc, batch):
    a = u8img(*shape, seed=shape[0] + rr, batch=batch)
    y = libsat.box_filter(dev(a), rr, rc)
    assert libsat.last_launch_count() == 1          # fused: one launch, no SAT in HBM
    got = y.cpu().numpy()
    for b in range(batch):
        assert np.array_equal(got[b], oracle.box_filter(a[b].astype(np.int32), rr, rc)), b


@pytest.mark.parametrize("rr,rc", [(1, 1), (16, 33), (5, 127)])
def test_box_fused_int32_wrapping(libsat, rr, rc):
    a = make_np(700, 1000, "int32", "u32", seed=rr + rc, batch=2)
    y = libsat.box_filter(dev(a), rr, rc)
    assert libsat.last_launch_count() == 1
    got = y.cpu().numpy()
    for b in range(2):
        assert np.array_equal(got[b], oracle.box_filter(a[b], rr, rc))


@pytest.mark.parametrize("normalize", [False, True])
@pytest.mark.parametrize("rr,rc", [(4, 6), (8, 127), (0, 2)])
def test_box_fused_float32(libsat, normalize, rr, rc):
    """float32 input, float64 SAT on chip; dyadic inputs make every box sum
    exact, so both output types match the correctly rounded oracle value."""
    a = make_np(333, 1000, "float32", "unit", seed=rr * 7 + rc, batch=2)
    for out_dtype in (torch.float32, torch.float64):
        y = libsat.box_filter(dev(a), rr, rc, normalize=normalize, out_dtype=out_dtype)
        assert libsat.last_launch_count() == 1
        got = y.cpu().numpy()
        for b in range(2):
            ref = oracle.box_filter(a[b], rr, rc, normalize=normalize)
            assert np.array_equal(got[b], ref.astype(got.dtype))


def test_box_fused_matches_two_pass(libsat):
    """The fused kernel and the two-pass path (forced by in-place output) agree
    bit for bit; a radius beyond the fused limit takes the two-pass path."""
    a = make_np(540, 960, "int32", "u32", seed=3)
    x = dev(a)
    fused = libsat.box_filter(x, 5, 9).cpu().numpy()
    assert libsat.last_launch_count() == 1
    y = x.clone()
    libsat.box_filter(y, 5, 9, out=y)
    assert libsat.last_launch_count() >= 2
    assert np.array_equal(fused, y.cpu().numpy())
    big = libsat.box_filter(x, 40, 3).cpu().numpy()
    assert libsat.last_launch_count() >= 2
    assert np.array_equal(big, oracle.box_filter(a, 40, 3))


def test_box_huge_radius_clamped(libsat):
    """a radius of INT_MAX ('the whole image') is clamped on the
    host; every window covers the whole image, so every output is the image
    total (mod 2^32)."""
    a = u8img(300, 500, seed=12, batch=2)
    y = libsat.box_filter(dev(a), 2**31 - 1, 2**31 - 1).cpu().numpy()
    for b in range(2):
        assert (y[b] == np.int64(a[b].astype(np.int64).sum()).astype(np.int32)).all()
        assert np.array_equal(y[b], oracle.box_filter(a[b].astype(np.int32), 300, 500))


@pytest.mark.parametrize("rb", [1, 5, 17, 64, 200])
def test_box_walk_row_blocks(libsat, rb):
    """Column-walk box filter with forced rows per unit:
    every unit re-runs the 2 rr-row warm-up of its window, so unit borders
    anywhere (1 row, ragged, taller than the image) give the same sums."""
    try:
        libsat.set_box_rows(rb)
        a = u8img(301, 520, seed=rb, batch=2)
        for rr, rc in ((0, 0), (4, 4), (8, 63), (3, 17)):
            y = libsat.box_filter(dev(a), rr, rc).cpu().numpy()
            assert libsat.last_launch_count() == 1
            for b in range(2):
                assert np.array_equal(y[b], oracle.box_filter(a[b].astype(np.int32), rr, rc)), (rr, rc, b)
        ai = make_np(150, 264, "int32", "u32", seed=rb, batch=2)
        y = libsat.box_filter(dev(ai), 6, 40).cpu().numpy()
        for b in range(2):
            assert np.array_equal(y[b], oracle.box_filter(ai[b], 6, 40))
    finally:
        libsat.set_box_rows(0)
