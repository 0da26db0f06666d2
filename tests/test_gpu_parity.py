"""GPU parity: libsat (through the C ABI) vs the CPU oracle, element by element.

int32: bit-exact (mod 2^32).  float32: max relative error <= 1e-5 against the
float64 oracle with inputs in [0, 1) (north star (5)).
Inputs are seeded and synthetic (sat_inputs); expected values come only from
``oracle``.  Run on a B200 via gpurun: ``pytest -m gpu``.
"""
import numpy as np
import pytest
import torch

import oracle
from sat_inputs import make_np, make_torch

pytestmark = pytest.mark.gpu

VARIANTS = ["1r1w", "2r2w", "2r1w", "1+rr1w"]
FTOL = 1e-5


@pytest.fixture(scope="module")
def libsat():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icpp_kasagini14_b200 as m
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def check(got, ref, dtype):
    got = got.cpu().numpy() if isinstance(got, torch.Tensor) else got
    if dtype == "int32":
        if not np.array_equal(got, ref):
            bad = np.argwhere(got != ref)
            raise AssertionError(f"{len(bad)} mismatches, first at {bad[:5].tolist()}")
    else:
        err = oracle.max_rel_err(got, ref)
        assert err <= FTOL, f"max rel err {err}"


def gen(n, m, dtype, seed=1):
    return make_np(n, m, dtype, "u32" if dtype == "int32" else "unit", seed=seed)


# ------------------------------------------------------------------ worked example
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_fig3(libsat, fig3, variant, dtype):
    a, _, b = fig3
    x = dev(a.astype(dtype))
    y = libsat.sat(x, variant=variant)
    assert np.array_equal(y.cpu().numpy(), b.astype(dtype))


# ------------------------------------------------------------------ shapes x variants
SHAPES = [(1, 1), (1, 5), (5, 1), (3, 5), (15, 127), (16, 128), (17, 129), (63, 255),
          (64, 256), (65, 257), (127, 129), (200, 1000), (1080, 1920), (333, 1001),
          (1000, 4096), (2049, 513)]


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("dtype", ["int32", "float32"])
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: f"{s[0]}x{s[1]}")
def test_shapes(libsat, variant, dtype, shape):
    a = gen(*shape, dtype, seed=shape[0] * 7 + shape[1])
    ref = oracle.sat(a)
    check(libsat.sat(dev(a), variant=variant), ref, dtype)


@pytest.mark.parametrize("tile_rows", [16, 32, 64, 128])
@pytest.mark.parametrize("generic", [False, True])
@pytest.mark.parametrize("variant", VARIANTS)
def test_tile_configs(libsat, tile_rows, generic, variant):
    for dtype in ("int32", "float32"):
        a = gen(700, 1300, dtype, seed=tile_rows)
        ref = oracle.sat(a)
        check(libsat.sat(dev(a), variant=variant, tile_rows=tile_rows, force_generic=generic),
              ref, dtype)
        if variant in ("1r1w", "2r1w", "1+rr1w") and not generic:
            assert libsat.last_tile_rows() == tile_rows


@pytest.mark.parametrize("r", [0.0, 0.1, 0.25, 0.5, 1.0])
def test_1plusr_r_sweep(libsat, r):
    a = gen(1500, 2000, "int32", seed=5)
    ref = oracle.sat(a)
    check(libsat.sat(dev(a), variant="1+rr1w", r=r, tile_rows=32), ref, "int32")
    re = libsat.last_r_effective()
    assert abs(re - r) < 0.15


def test_in_place(libsat):
    for variant in VARIANTS:
        a = gen(517, 777, "int32", seed=3)
        ref = oracle.sat(a)
        x = dev(a)
        y = libsat.sat(x, variant=variant, out=x)
        assert y.data_ptr() == x.data_ptr()
        check(x, ref, "int32")


def test_input_not_modified(libsat):
    a = gen(300, 400, "float32", seed=2)
    x = dev(a)
    for variant in VARIANTS:
        libsat.sat(x, variant=variant)
        assert np.array_equal(x.cpu().numpy(), a)


def test_closed_forms(libsat):
    n, m = 1024, 3000
    ones = torch.ones(n, m, dtype=torch.int32, device="cuda")
    i = np.arange(n, dtype=np.int64)[:, None] + 1
    j = np.arange(m, dtype=np.int64)[None, :] + 1
    for variant in VARIANTS:
        got = libsat.sat(ones, variant=variant).cpu().numpy().astype(np.int64)
        assert np.array_equal(got, i * j), variant
    # float32 all-ones is exact while the SAT <= 2^24
    f = torch.ones(2048, 2048, dtype=torch.float32, device="cuda")
    for variant in VARIANTS:
        got = libsat.sat(f, variant=variant).cpu().numpy()
        assert np.array_equal(got, (np.arange(1, 2049)[:, None] * np.arange(1, 2049)[None, :]).astype(np.float32))


def test_repeated_calls_fresh_tags(libsat):
    """Descriptors are never cleared between calls: per-launch tags must keep
    stale words from being taken (SURVEY 7 'flag reset between calls')."""
    for k in range(40):
        shape = (300 + 37 * k, 200 + 91 * k)
        a = gen(*shape, "int32", seed=100 + k)
        check(libsat.sat(dev(a)), oracle.sat(a), "int32")
        assert libsat.last_launch_count() == 1


def test_lookback_jitter_stress(libsat):
    for th in (16, 32, 64, 128):
        a = gen(3000, 2500, "int32", seed=th)
        check(libsat.sat(dev(a), tile_rows=th, jitter=20000), oracle.sat(a), "int32")
        af = gen(3000, 2500, "float32", seed=th)
        check(libsat.sat(dev(af), tile_rows=th, jitter=20000), oracle.sat(af), "float32")


def test_int32_deterministic(libsat):
    a = dev(gen(4096, 4096, "int32", seed=9))
    r1 = libsat.sat(a).cpu()
    for _ in range(3):
        assert torch.equal(libsat.sat(a).cpu(), r1)


# ------------------------------------------------------------------ batch / seeded / sharded
@pytest.mark.parametrize("variant", VARIANTS)
def test_batched(libsat, variant):
    for dtype in ("int32", "float32"):
        a = make_np(130, 300, dtype, "u32" if dtype == "int32" else "unit", seed=4, batch=5)
        y = libsat.sat_batched(dev(a), variant=variant).cpu().numpy()
        for b in range(5):
            check(y[b], oracle.sat(a[b]), dtype)


def test_batched_images_cfg5_slice(libsat):
    a = make_np(1080, 1920, "float32", "unit", seed=77, batch=4)
    y = libsat.sat_batched(dev(a)).cpu().numpy()
    for b in range(4):
        check(y[b], oracle.sat(a[b]), "float32")
    assert libsat.last_launch_count() == 1


def test_seeded(libsat):
    for dtype in ("int32", "float32"):
        full = gen(900, 1100, dtype, seed=8)
        ref = oracle.sat(full)
        r0 = 311
        strip = dev(full[r0:])
        if dtype == "int32":
            carry = oracle.column_totals(full[:r0])
        else:
            carry = full[:r0].astype(np.float64).sum(axis=0).astype(np.float32)
        check(libsat.sat_seeded(strip, carry_row=dev(carry)), ref[r0:], dtype)
        check(libsat.sat_seeded(strip, sat_row=dev(ref[r0 - 1].astype(dtype))), ref[r0:], dtype)


def test_column_totals_and_exscan(libsat):
    for dtype in ("int32", "float32"):
        a = gen(5000, 1234, dtype, seed=6)
        t = libsat.column_totals(dev(a)).cpu().numpy()
        ref = oracle.column_totals(a)
        if dtype == "int32":
            assert np.array_equal(t, ref)
        else:
            assert np.max(np.abs(t - ref) / np.maximum(ref, 1e-30)) < 1e-5
        g = gen(6, 1234, dtype, seed=7)
        for rank in range(6):
            e = libsat.rank_exscan(dev(g), rank).cpu().numpy()
            r = oracle.rank_exscan(g, rank)
            if dtype == "int32":
                assert np.array_equal(e, r)
            else:
                assert np.allclose(e, r, rtol=1e-6, atol=0)


def test_seeded_gathered_is_the_rank_exscan(libsat):
    """sat_compute_seeded_sum: band 0 adds sum_{q<rank} gathered[q] to its
    first row (the sharded mode's exclusive scan inside the SAT kernel), for
    every rank, in one launch."""
    P, n, m = 5, 640, 1100
    for dtype in ("int32", "float32"):
        full = gen(n, m, dtype, seed=17)
        ref = oracle.sat(full)
        r0 = 257
        if dtype == "int32":
            above = oracle.column_totals(full[:r0])
        else:
            above = full[:r0].astype(np.float64).sum(axis=0)
        # P gathered vectors whose prefix of length `rank` sums to `above`
        rng = np.random.default_rng(3)
        for rank in range(1, P + 1):
            g = np.zeros((P, m), dtype=np.float64 if dtype == "float32" else np.uint32)
            if dtype == "int32":
                parts = rng.integers(0, 2**32, size=(rank - 1, m), dtype=np.uint64).astype(np.uint32)
                with np.errstate(over="ignore"):
                    last = above.view(np.uint32) - parts.sum(axis=0, dtype=np.uint32)
                g[:rank - 1] = parts
                g[rank - 1] = last
                gd = dev(g.view(np.int32))
            else:
                g[:rank] = above / rank
                gd = dev(g.astype(np.float32))
            got = libsat.sat_seeded(dev(full[r0:]), gathered=gd, rank=rank)
            assert libsat.last_launch_count() == 1
            check(got, ref[r0:], dtype)


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("variant", ["1r1w", "2r2w"])
def test_sharded_abi_variants(libsat, P, variant):
    """sat_compute_sharded_ex: the 2R2W strip takes the carry row in its column
    pass; same strips as the unsharded SAT."""
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    n, m = 1500, 1000
    for dtype in ("int32", "float32"):
        full = gen(n, m, dtype, seed=P + 11)
        ref = oracle.sat(full)
        bounds = [partition_rows(n, P, p) for p in range(P)]
        strips = [dev(full[r0:r1]) for r0, r1 in bounds]
        totals = [libsat.column_totals(s) for s in strips]
        totals[-1] = torch.zeros_like(totals[-1])
        outs = []
        for p in range(P):
            def ag(send, recv, p=p):
                torch.cuda.synchronize()
                recv.copy_(torch.stack(totals))
            o, st = libsat.sat_sharded_abi(strips[p], p, P, ag, variant=variant)
            outs.append(o.cpu().numpy())
            rows = bounds[p][1] - bounds[p][0]
            assert st["strip_bytes_read"] == rows * m * 4 * (2 if variant == "2r2w" else 1)
        check(np.concatenate(outs), ref, dtype)


@pytest.mark.parametrize("variant", ["1r1w", "2r2w"])
def test_sharded_nccl_single_rank(libsat, variant):
    """In-library NCCL communicator (sat_nccl_comm_create, sat_compute_sharded_nccl)
    with one rank: libnccl loaded, communicator created on the device, rank and
    size read back from it, the strip computed.  NCCL refuses two ranks on one
    device, and a one-rank strip needs no gather, so ncclAllGather itself only
    runs with >= 2 GPUs (bench.py --exchange libsat-nccl); the gather callback
    path it plugs into is the one the virtual-rank tests above exercise."""
    comm = libsat.NcclComm(libsat.nccl_unique_id(), 0, 1)
    try:
        for dtype in ("int32", "float32"):
            a = gen(1000, 1300, dtype, seed=21)
            y, st = libsat.sat_sharded_nccl(dev(a), comm, variant=variant)
            check(y, oracle.sat(a), dtype)
            assert st["extra_bytes_read"] == 0 and st["allgather_bytes"] == 0
    finally:
        comm.close()


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_sharded_abi_single_process(libsat, P):
    """sat_compute_sharded with a fake all-gather: P ranks simulated one after
    another on one GPU; the concatenated strips must equal the unsharded SAT."""
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    n, m = 2000, 1500
    for dtype in ("int32", "float32"):
        full = gen(n, m, dtype, seed=P)
        ref = oracle.sat(full)
        bounds = [partition_rows(n, P, p) for p in range(P)]
        strips = [dev(full[r0:r1]) for r0, r1 in bounds]
        totals = [libsat.column_totals(s) for s in strips]
        totals[-1] = torch.zeros_like(totals[-1])
        outs = []
        for p in range(P):
            def ag(send, recv, p=p):
                torch.cuda.synchronize()
                assert torch.equal(send, totals[p])
                recv.copy_(torch.stack(totals))
            o, st = libsat.sat_sharded_abi(strips[p], p, P, ag)
            outs.append(o.cpu().numpy())
            # one totals launch (ranks < P-1) + one SAT launch
            assert libsat.last_launch_count() == (2 if (P > 1 and p < P - 1) else 1)
            rows = bounds[p][1] - bounds[p][0]
            assert st["extra_bytes_read"] == (rows * m * 4 if (P > 1 and p < P - 1) else 0)
        check(np.concatenate(outs), ref, dtype)


# ------------------------------------------------------------------ host e2e
@pytest.mark.parametrize("pinned", [True, False])
def test_host_end_to_end(libsat, pinned):
    for dtype in ("int32", "float32"):
        a = gen(3000, 2048, dtype, seed=12)
        x = torch.from_numpy(a)
        if pinned:
            x = x.pin_memory()
        y = libsat.sat_host(x)
        check(y.numpy(), oracle.sat(a), dtype)


# ------------------------------------------------------------------ BASELINE.json configs
def test_cfg1_1024_int32(libsat):
    a = gen(1024, 1024, "int32", seed=1001)
    check(libsat.sat(dev(a)), oracle.sat(a), "int32")


@pytest.mark.parametrize("variant", VARIANTS)
def test_cfg2_4096_float32(libsat, variant):
    a = gen(4096, 4096, "float32", seed=2001)
    check(libsat.sat(dev(a), variant=variant), oracle.sat(a), "float32")


@pytest.mark.slow
@pytest.mark.parametrize("n", [16384, 18432])
def test_cfg3_full_int32(libsat, n):
    """Full-size parity in the launch configuration bench.py times."""
    x = make_torch(n, n, "int32", "u32", seed=3001, device="cuda")
    y = libsat.sat(x).cpu().numpy()
    a = x.cpu().numpy()
    del x
    st = oracle.Stream(n, True)
    step = 2048
    for r0 in range(0, n, step):
        ref = st.feed(a[r0:r0 + step])
        assert np.array_equal(y[r0:r0 + step], ref), f"rows {r0}.."


@pytest.mark.slow
def test_cfg3_float32_16k(libsat):
    n = 16384
    x = make_torch(n, n, "float32", "unit", seed=3002, device="cuda")
    y = libsat.sat(x).cpu().numpy()
    a = x.cpu().numpy()
    st = oracle.Stream(n, False)
    worst = 0.0
    for r0 in range(0, n, 2048):
        ref = st.feed(a[r0:r0 + 2048])
        worst = max(worst, oracle.max_rel_err(y[r0:r0 + 2048], ref))
    assert worst <= FTOL, worst


@pytest.mark.slow
def test_cfg4_65536_properties(libsat):
    """64K x 64K int32 (16 GiB): closed form on all-ones (wrap pins:
    b[65535][65535] = 0, b[32767][65535] = INT32_MIN) and sampled exact
    elements of a random matrix via the oracle's one-element sum."""
    n = 65536
    x = torch.ones(n, n, dtype=torch.int32, device="cuda")
    libsat.sat(x, out=x)
    assert int(x[65535, 65535]) == 0
    assert int(x[32767, 65535]) == -2**31
    for r in (0, 1, 4095, 30000, 65535):
        row = x[r].cpu().numpy().view(np.uint32).astype(np.int64)
        assert np.array_equal(row, ((r + 1) * np.arange(1, n + 1, dtype=np.int64)) % 2**32)
    del x
    torch.cuda.empty_cache()
    x = make_torch(n, n, "int32", "u32", seed=4001, device="cuda")
    y = libsat.sat(x)
    torch.cuda.synchronize()
    # exact elements near the top-left (oracle one-element sums on a host block)
    blk = x[:512, :].cpu().numpy()
    for (i, j) in [(0, 0), (511, 65535), (300, 40000), (17, 65535)]:
        assert int(y[i, j]) == int(oracle.sat_at(blk, i, j))
    # inclusion-exclusion recovers the input on sampled 2x2 windows everywhere
    rng = np.random.default_rng(0)
    for _ in range(200):
        i = int(rng.integers(1, n)); j = int(rng.integers(1, n))
        w = y[i - 1:i + 1, j - 1:j + 1].cpu().numpy().view(np.uint32)
        with np.errstate(over="ignore"):
            rec = w[1, 1] - w[0, 1] - w[1, 0] + w[0, 0]
        assert rec == np.uint32(int(x[i, j]) & 0xFFFFFFFF)
    # the LAST 2048 rows, whole, against the oracle streamed from the column
    # sums of every row above them: these rows are the end of the longest
    # vertical carry chain (511 bands, 16 segments), which the 2x2 windows
    # above cannot see (they cancel any per-band carry error).  The column
    # sums come from torch (int64 accumulation of the input rows, independent
    # of libsat); the SAT rows from the oracle.
    r0 = n - 2048
    acc = torch.zeros(n, dtype=torch.int64, device="cuda")
    for a in range(0, r0, 4096):
        acc += x[a:min(r0, a + 4096)].to(torch.int64).sum(dim=0)
    st = oracle.Stream(n, True)
    st.colsum[:] = (acc % 2**32).cpu().numpy().astype(np.uint32)
    for a in range(r0, n, 512):
        ref = st.feed(x[a:a + 512].cpu().numpy())
        got = y[a:a + 512].cpu().numpy()
        assert np.array_equal(got, ref), f"rows {a}..{a + 511}"


def test_float_nan_inf_propagate(libsat):
    """IEEE semantics: a NaN poisons every SAT element at or
    below-right of it, +Inf likewise (no FTZ / fast-math), for every variant;
    elements above or left of it stay finite and exact."""
    for dtype in ("float32", "float64"):
        a = make_np(600, 700, dtype, "unit", seed=1)
        a[300, 400] = np.nan
        a[100, 650] = np.inf
        for variant in VARIANTS:
            got = libsat.sat(dev(a), variant=variant).cpu().numpy()
            assert np.isnan(got[300:, 400:]).all(), variant
            assert np.isinf(got[100:300, 650:]).all() and (got[100:300, 650:] > 0).all(), variant
            clean = a.copy()
            clean[300, 400] = 0
            clean[100, 650] = 0
            ref = oracle.sat(clean)
            ok = np.isfinite(got)
            assert ok[:100].all() and ok[:300, :400].all()
            if dtype == "float64":
                assert np.array_equal(got[:300, :400], ref[:300, :400]), variant
            else:
                assert oracle.max_rel_err(got[:300, :400], ref[:300, :400]) <= FTOL, variant


def test_debug_trace_records_events(libsat):
    """Event traces exist in debug builds only (SAT_DEBUG=1); the release
    library refuses them loudly."""
    if libsat.lib.sat_debug_trace(None) != 0:
        with pytest.raises(Exception, match="debug build"):
            libsat.debug_trace(torch.zeros(8, dtype=torch.int64, device="cuda"))
        return
    a = gen(640, 1024, "int32", seed=44)
    x = dev(a)
    nb, nc = 10, 8
    buf = torch.zeros(nb * nc * 8, dtype=torch.int64, device="cuda")
    libsat.debug_trace(buf)
    y = libsat.sat(x, tile_rows=64)
    torch.cuda.synchronize()
    check(y, oracle.sat(a), "int32")
    t = buf.view(nb, nc, 8).cpu().numpy()
    assert (t[:, :, 0] != 0).all() and (t[:, :, 2] != 0).all()
    assert libsat.last_grid() >= 1


@pytest.mark.parametrize("shape", [(64 * 600 + 7, 256), (64 * 640, 777 * 4)])
def test_big_ring_config(libsat, shape):
    """TH=64 with one CTA per SM and 1-KB row segments per TMA load (chosen
    automatically for >= 4 waves of TH-64 bands)."""
    for dtype in ("int32", "float32"):
        a = gen(*shape, dtype, seed=shape[0])
        check(libsat.sat(dev(a), tile_rows=64), oracle.sat(a), dtype)


@pytest.mark.parametrize("nseg", [2, 3, 7])
@pytest.mark.parametrize("tile_rows", [64, 128])
def test_band_segments(libsat, nseg, tile_rows):
    """Band segments: a ticket is (segment, band) and the
    row carry crosses segments through tagged words; every split is exact."""
    kw = dict(tile_rows=tile_rows, segments=nseg)
    for shape in [(1000, 1300), (64 * 40 + 7, 2048), (300, 777 * 4)]:
        for dtype in ("int32", "float32"):
            a = gen(*shape, dtype, seed=nseg * 7 + shape[0])
            check(libsat.sat(dev(a), **kw), oracle.sat(a), dtype)
    a = gen(3 * 400, 1920, "int32", seed=5).reshape(3, 400, 1920)
    got = libsat.sat_batched(dev(a), **kw).cpu().numpy()
    for i in range(3):
        assert np.array_equal(got[i], oracle.sat(a[i]))
    # repeated calls reuse the carry buffer with fresh tags; jitter shuffles timing
    x = dev(gen(2048, 4096, "int32", seed=3))
    ref = oracle.sat(x.cpu().numpy())
    for _ in range(3):
        check(libsat.sat(x, **kw), ref, "int32")
    check(libsat.sat(x, jitter=20000, **kw), ref, "int32")


@pytest.mark.parametrize("nseg", [3, 4, 5])
@pytest.mark.parametrize("tile_rows", [64, 128])
def test_unit_queue_many_units(libsat, nseg, tile_rows):
    """Many short units per CTA: the next unit's loads
    start before the current unit's control groups are done, so a group's
    chunks must stay G apart across unit boundaries.  Segments of a number of
    chunks that is not a multiple of the control-group count (3 at TH 112/128)
    failed before the assignment became CTA-global."""
    kw = dict(tile_rows=tile_rows, segments=nseg)
    a = gen(20000, 3000, "int32", seed=nseg + tile_rows)
    ref = oracle.sat(a)
    x = dev(a)
    check(libsat.sat(x, **kw), ref, "int32")
    check(libsat.sat(x, jitter=20000, **kw), ref, "int32")
    af = gen(9000, 2500, "float32", seed=nseg)
    check(libsat.sat(dev(af), **kw), oracle.sat(af), "float32")
    # 65536 x 4096 all ones, in place (1 GiB): 2048 units of 8 chunks at nseg 4
    if nseg == 4:
        n, m = 65536, 4096
        y = torch.ones(n, m, dtype=torch.int32, device="cuda")
        libsat.sat(y, out=y, **kw)
        jj = torch.arange(1, m + 1, device="cuda", dtype=torch.int64)
        for r in (0, 127, 17664, 18944, 40000, n - 1):
            assert torch.equal(y[r].to(torch.int64) % 2**32, ((r + 1) * jj) % 2**32), r
        assert int(y[n - 1, m - 1]) == (n * m) % 2**32 - (2**32 if (n * m) % 2**32 >= 2**31 else 0)


# ------------------------------------------------------------------ 4R4W / 4R1W
PAPER_VARIANTS = ["4r4w", "4r1w"]


def check_4r1w_f32(got, a):
    """4R1W in float32: Formula (1) subtracts, so rounding errors do not stay
    relative.  The computed b-hat satisfies b-hat = a + b-hat_up + b-hat_left
    - b-hat_diag + delta with |delta_ij| <= 3u (2 b_ij + 1) for inputs in
    [0, 1) (three roundings of partial sums <= 2 b_ij + 1, u = 2^-24), and the
    error e = b-hat - b obeys the same recurrence, so e = SAT(delta) and
    |e_ij| <= 3u SAT(2b + 1)_ij (R16).  Checked element by element
    (with 1 % slack for second-order terms)."""
    ref = oracle.sat(a)
    bound = 3 * 2.0 ** -24 * np.cumsum(np.cumsum(2 * ref + 1, axis=0), axis=1) * 1.01
    err = np.abs(got.astype(np.float64) - ref)
    assert (err <= bound).all(), f"max err/bound {(err / bound).max()}"


@pytest.mark.parametrize("variant", PAPER_VARIANTS)
@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_fig3_paper_variants(libsat, fig3, variant, dtype):
    a, _, b = fig3
    y = libsat.sat(dev(a.astype(dtype)), variant=variant)
    assert np.array_equal(y.cpu().numpy(), b.astype(dtype))


@pytest.mark.parametrize("variant", PAPER_VARIANTS)
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: f"{s[0]}x{s[1]}")
def test_shapes_paper_variants(libsat, variant, shape):
    a = gen(*shape, "int32", seed=shape[0] * 3 + shape[1])
    check(libsat.sat(dev(a), variant=variant), oracle.sat(a), "int32")
    af = gen(*shape, "float32", seed=shape[0] * 3 + shape[1])
    got = libsat.sat(dev(af), variant=variant).cpu().numpy()
    if variant == "4r4w":
        check(got, oracle.sat(af), "float32")
    else:
        check_4r1w_f32(got, af)


@pytest.mark.parametrize("variant", PAPER_VARIANTS)
def test_paper_variants_inplace_batched(libsat, variant):
    a = gen(3 * 129, 200, "int32", seed=9).reshape(3, 129, 200)
    got = libsat.sat_batched(dev(a), variant=variant).cpu().numpy()
    for i in range(3):
        assert np.array_equal(got[i], oracle.sat(a[i]))
    b = gen(257, 300, "int32", seed=10)
    x = dev(b)
    y = libsat.sat(x, variant=variant, out=x)
    assert y.data_ptr() == x.data_ptr()
    assert np.array_equal(x.cpu().numpy(), oracle.sat(b))


def test_4r4w_cfg2_and_4r1w_4096(libsat):
    af = gen(4096, 4096, "float32", seed=2)
    check(libsat.sat(dev(af), variant="4r4w"), oracle.sat(af), "float32")
    a = gen(4096, 4096, "int32", seed=2)
    check(libsat.sat(dev(a), variant="4r1w"), oracle.sat(a), "int32")
    assert libsat.last_launch_count() == 4096 + 4096 - 1


# ------------------------------------------------------------------ fused peer exchange
@pytest.mark.parametrize("P", [2, 3, 8])
@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
def test_fused_exchange_single_device(libsat, P, dtype):
    """P virtual ranks on one GPU, each on its own stream with its own mailbox
    (the peer pointers are plain device pointers instead of IPC mappings --
    the kernels and the flag/acknowledge protocol are the same).  Several
    consecutive calls reuse both mailbox parities without any barrier; every
    call must equal the unsharded SAT (bit-exact for int32 / dyadic float64)."""
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    tdt = {"int32": torch.int32, "float32": torch.float32, "float64": torch.float64}[dtype]
    n, m = 1500, 1300
    nb = libsat.PeerExchange.mailbox_bytes(m, P, tdt)
    boxes = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(P)]
    ptrs = [b.data_ptr() for b in boxes]
    exs = [libsat.PeerExchange(p, P, m, tdt, boxes[p], ptrs) for p in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    bounds = [partition_rows(n, P, p) for p in range(P)]
    for it in range(5):
        full = make_np(n, m, dtype, "u32" if dtype == "int32" else "unit", seed=it)
        ref = oracle.sat(full)
        strips = [dev(full[a:b]) for a, b in bounds]
        outs = [torch.empty_like(s) for s in strips]
        torch.cuda.synchronize()
        for p in range(P):
            with torch.cuda.stream(streams[p]):
                exs[p].sat(strips[p], out=outs[p], stream=streams[p])
        torch.cuda.synchronize()
        got = np.concatenate([o.cpu().numpy() for o in outs])
        if dtype == "float32":
            check(got, ref, "float32")
        else:
            assert np.array_equal(got, ref), f"call {it}"
    for e in exs:
        e.close()


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("shape,dtype", [((512, 1024), "int32"), ((1000, 3000), "float32"),
                                         ((4096, 4096), "int32")])
def test_cuda_graph_replay(libsat, variant, shape, dtype):
    """Captured SAT calls replay correctly: the look-back ticket base comes
    from the device, so every replay, and every eager call
    on the same stream after it, sees fresh tags.  New input contents are
    copied into the captured buffer between replays."""
    n, m = shape
    x = dev(gen(n, m, dtype, seed=1))
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        y = libsat.sat(x, variant=variant)          # warm: sizes the workspace of stream s
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.sat(x, variant=variant, out=y)
    for it in range(4):
        host = gen(n, m, dtype, seed=10 + it)
        x.copy_(dev(host))
        g.replay()
        torch.cuda.synchronize()
        check(y.cpu().numpy(), oracle.sat(host), dtype)
        with torch.cuda.stream(s):                  # eager call between replays
            z = libsat.sat(x, variant=variant)
        s.synchronize()
        check(z.cpu().numpy(), oracle.sat(host), dtype)


def test_cuda_graph_batched_two_shapes(libsat):
    """Two captured calls of different shapes on one stream (batched and 2-D),
    one graph, the workspace sized by eager calls of both."""
    a = gen(700, 1500, "int32", seed=7)
    xb = dev(make_np(300, 800, "int32", "u32", seed=8, batch=5))
    x = dev(a)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        y = libsat.sat(x)
        yb = libsat.sat_batched(xb)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.sat(x, out=y)
        libsat.sat_batched(xb, out=yb)
    for it in range(3):
        a = gen(700, 1500, "int32", seed=60 + it)
        ab = make_np(300, 800, "int32", "u32", seed=70 + it, batch=5)
        x.copy_(dev(a))
        xb.copy_(dev(ab))
        g.replay()
        torch.cuda.synchronize()
        check(y, oracle.sat(a), "int32")
        got = yb.cpu().numpy()
        for b in range(5):
            check(got[b], oracle.sat(ab[b]), "int32")


@pytest.mark.parametrize("space,replays", [("300000", 6), ("540000", 60)])
def test_cuda_graph_tag_reset(libsat, space, replays):
    """A tiny tag space (sat_debug_set_tag_space) makes sat_epoch_kernel clear the
    descriptors on every replay (each launch's value range crosses a multiple
    of half the space), and forces the host-side reset on eager calls of a
    never-captured stream.  At 540000 (half the space just above the
    per-launch bound) only some replays clear: the mixed regime."""
    libsat.set_tag_space(int(space))
    try:
        _graph_tag_reset(libsat, replays)
    finally:
        libsat.set_tag_space(0)


def _graph_tag_reset(libsat, replays):
    x = dev(gen(2048, 2048, "int32", seed=3))
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        y = libsat.sat(x)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.sat(x, out=y)
    for it in range(replays):
        host = gen(2048, 2048, "int32", seed=20 + it)
        x.copy_(dev(host))
        g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy(), oracle.sat(host)), f"replay {it}"
    host = gen(2048, 2048, "int32", seed=40)
    x2 = dev(host)
    for it in range(3):
        assert np.array_equal(libsat.sat(x2).cpu().numpy(), oracle.sat(host)), f"eager {it}"
        with torch.cuda.stream(s):
            z = libsat.sat(x2)
        s.synchronize()
        assert np.array_equal(z.cpu().numpy(), oracle.sat(host)), f"eager after capture {it}"


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")
def test_capture_cold_workspace_refused(libsat):
    """Capturing on a stream whose workspace was never sized fails loudly
    (a captured call cannot allocate)."""
    x = dev(gen(640, 1280, "int32", seed=5))
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with pytest.raises(Exception, match="warm workspace"):
        with torch.cuda.graph(g, stream=s):
            libsat.sat(x)
    torch.cuda.synchronize()
    check(libsat.sat(x), oracle.sat(x.cpu().numpy()), "int32")


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")
def test_capture_host_call_refused(libsat):
    """sat_host synchronizes its stream, so it refuses capture loudly."""
    a = torch.from_numpy(gen(256, 512, "int32", seed=9)).pin_memory()
    o = torch.empty_like(a).pin_memory()
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with pytest.raises(Exception, match="cannot be captured"):
        with torch.cuda.graph(g, stream=s):
            libsat.sat_host(a, o)
    torch.cuda.synchronize()
    libsat.sat_host(a, o)
    assert np.array_equal(o.numpy(), oracle.sat(a.numpy()))


def test_graph_replay_after_workspace_growth(libsat):
    """capture a small call, grow the stream's workspace
    with a larger eager call, replay the graph: the graph's buffers were
    retired (not freed), so the replay is still correct and writes nothing
    into memory the caller allocated afterwards; sat_release_workspace then
    frees everything and the stream starts over."""
    s = torch.cuda.Stream()
    a = gen(640, 1280, "int32", seed=61)
    x = dev(a)
    with torch.cuda.stream(s):
        y = libsat.sat(x)                    # sizes the workspace for this shape
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        libsat.sat(x, out=y)
    big = gen(4096, 4096, "int32", seed=62)
    with torch.cuda.stream(s):
        yb = libsat.sat(dev(big))            # grows the descriptors: old buffers retired
    s.synchronize()
    check(yb, oracle.sat(big), "int32")
    sentinel = torch.full((64 << 20,), 0x5A5A5A5A, dtype=torch.int32, device="cuda")
    for it in range(3):
        host = gen(640, 1280, "int32", seed=70 + it)
        x.copy_(dev(host))
        with torch.cuda.stream(s):
            g.replay()
        s.synchronize()
        check(y, oracle.sat(host), "int32")
    assert bool((sentinel == 0x5A5A5A5A).all())
    libsat.release_workspace(s)
    with torch.cuda.stream(s):
        z = libsat.sat(x)
    s.synchronize()
    check(z, oracle.sat(x.cpu().numpy()), "int32")


@pytest.mark.slow
def test_fused_exchange_with_band_segments(libsat):
    """Strips tall and wide enough for band segments (> one wave of TH-128
    bands, >= 32 chunks): every band-0 segment unit adds its columns' share of
    the peers' totals, and only the last one acknowledges (the self-resetting
    counter), over 4 consecutive calls (both parities) on 2 virtual ranks."""
    from paper_conf_icpp_kasagini14_b200.dist import partition_rows
    P, n, m = 2, 2 * 20480, 4096
    nb = libsat.PeerExchange.mailbox_bytes(m, P, torch.int32)
    boxes = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(P)]
    ptrs = [b.data_ptr() for b in boxes]
    exs = [libsat.PeerExchange(p, P, m, torch.int32, boxes[p], ptrs) for p in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    bounds = [partition_rows(n, P, p) for p in range(P)]
    for it in range(4):
        full = make_torch(n, m, "int32", "u32", seed=90 + it, device="cuda")
        strips = [full[a:b] for a, b in bounds]
        outs = [torch.empty_like(s) for s in strips]
        torch.cuda.synchronize()
        for p in range(P):
            with torch.cuda.stream(streams[p]):
                exs[p].sat(strips[p], out=outs[p], stream=streams[p])
        torch.cuda.synchronize()
        # rank 1's strip against the oracle streamed from torch column sums of rank 0's rows
        st = oracle.Stream(m, True)
        st.colsum[:] = (full[:bounds[1][0]].to(torch.int64).sum(dim=0) % 2**32).cpu().numpy().astype(np.uint32)
        r0 = bounds[1][0]
        for a in range(0, bounds[1][1] - r0, 4096):
            ref = st.feed(full[r0 + a:r0 + a + 4096].cpu().numpy())
            assert np.array_equal(outs[1][a:a + 4096].cpu().numpy(), ref), (it, a)
        check(outs[0][:512], oracle.sat(full[:512].cpu().numpy()), "int32")
    for e in exs:
        e.close()


@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_2r2w_th128_column_pass(libsat, dtype):
    """2R2W's column pass takes the TH-128 band configuration where plain 1R1W
    does (forced, and automatic at 16384 rows); the row pass stays at TH 64."""
    a = gen(3000, 2500, dtype, seed=31)
    check(libsat.sat(dev(a), variant="2r2w", tile_rows=128), oracle.sat(a), dtype)
    b = gen(16384, 1100, dtype, seed=32)
    check(libsat.sat(dev(b), variant="2r2w"), oracle.sat(b), dtype)
    check(libsat.sat(dev(b), variant="2r2w", jitter=20000), oracle.sat(b), dtype)


@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_2r1w_auto_th128(libsat, dtype):
    """2R1W takes TH 128 automatically where plain 1R1W does (16384 rows)."""
    a = gen(16384, 1000, dtype, seed=33)
    check(libsat.sat(dev(a), variant="2r1w"), oracle.sat(a), dtype)
    assert libsat.last_tile_rows() == 128
