"""Pins for the CPU oracle (``oracle/``) against things other than itself.

Every test here is CPU-only.  Each pin cites what fixes the expected value:
the paper's worked example (Fig. 3), brute force written out in pure Python,
closed forms, library routines (numpy cumsum) on special cases, and algebraic
invariants.  A dropped term, a wrong sign or index, an exclusive-vs-inclusive
slip or a transposed operand in the oracle fails at least one of them.
"""
import itertools

import numpy as np
import pytest

import oracle
from sat_inputs import make_np

FORMS = [oracle.sat, oracle.sat_eq1, oracle.sat_2pass]


def py_brute(a):
    """Pure-Python double sum (independent of the oracle's C code)."""
    n, m = len(a), len(a[0]) if len(a) else 0
    out = [[0] * m for _ in range(n)]
    for i in range(n):
        for j in range(m):
            s = 0
            for k in range(i + 1):
                for l in range(j + 1):
                    s += a[k][l]
            out[i][j] = s
    return out


def to_u32(x):
    return np.asarray(x, dtype=np.int32).view(np.uint32)


# ---------------------------------------------------------------- Fig. 3
@pytest.mark.parametrize("form", FORMS + [oracle.sat_brute])
def test_fig3_int(fig3, form):
    a, cp, b = fig3
    assert np.array_equal(form(a), b)


@pytest.mark.parametrize("form", FORMS + [oracle.sat_brute])
def test_fig3_float(fig3, form):
    a, cp, b = fig3
    assert np.array_equal(form(a.astype(np.float32)), b.astype(np.float64))


def test_fig3_golden_self_consistent(fig3):
    """The recovered figure panels obey P:L193 (library cumsum, not oracle)."""
    a, cp, b = fig3
    assert np.array_equal(np.cumsum(a, axis=0), cp)
    assert np.array_equal(np.cumsum(cp, axis=1), b)
    assert b[0, 3] == a[0, 3] == 1          # inclusive (reading R1)
    assert b[8, 8] == a.sum() == 71


# ---------------------------------------------------------------- brute force
@pytest.mark.parametrize("n,m", [(n, m) for n in range(1, 7) for m in range(1, 7)])
def test_brute_small_int(n, m):
    rng = np.random.default_rng(n * 100 + m)
    a = rng.integers(-2**31, 2**31, size=(n, m), dtype=np.int64).astype(np.int32)
    ref = py_brute(a.astype(np.int64).tolist())
    ref = np.array(ref, dtype=np.int64) % (1 << 32)
    for form in FORMS + [oracle.sat_brute]:
        got = form(a).view(np.uint32).astype(np.int64)
        assert np.array_equal(got, ref), form.__name__


@pytest.mark.parametrize("n,m", [(1, 1), (3, 5), (5, 3), (7, 2), (13, 11)])
def test_brute_small_float(n, m):
    rng = np.random.default_rng(7 + n * m)
    a = rng.random((n, m)).astype(np.float32)
    from fractions import Fraction
    af = [[Fraction(float(x)) for x in row] for row in a]
    ref = py_brute(af)
    for form in FORMS + [oracle.sat_brute]:
        got = form(a)
        for i in range(n):
            for j in range(m):
                assert abs(Fraction(float(got[i, j])) - ref[i][j]) <= Fraction(1, 2**40) * (1 + abs(ref[i][j]))


def test_brute_random_64():
    rng = np.random.default_rng(3)
    a = rng.integers(0, 1000, size=(24, 31)).astype(np.int32)
    ref = np.array(py_brute(a.astype(np.int64).tolist()))
    assert np.array_equal(oracle.sat(a).astype(np.int64), ref)


# ---------------------------------------------------------------- rectangles
def test_rectangle_sums_all():
    """Sum of any rectangle = 4 SAT reads, every rectangle."""
    rng = np.random.default_rng(11)
    a = rng.integers(-50, 50, size=(9, 12)).astype(np.int32)
    b = oracle.sat(a)
    for r0, r1 in itertools.combinations_with_replacement(range(9), 2):
        for c0, c1 in itertools.combinations_with_replacement(range(12), 2):
            direct = int(a[r0:r1 + 1, c0:c1 + 1].astype(np.int64).sum()) % (1 << 32)
            assert int(oracle.rect_sum(b, r0, c0, r1, c1)) == direct


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n,m", [(1, 1), (37, 53), (53, 37), (1, 1000), (1000, 1), (129, 257)])
def test_all_ones_closed_form(n, m):
    a = np.ones((n, m), dtype=np.int32)
    i = np.arange(n)[:, None] + 1
    j = np.arange(m)[None, :] + 1
    ref = (i * j).astype(np.int64)
    for form in FORMS:
        assert np.array_equal(form(a).astype(np.int64), ref)
    assert np.array_equal(oracle.sat(a.astype(np.float32)), ref.astype(np.float64))


def test_int32_wrap_closed_form():
    """a = 2^16 everywhere => b = 2^16 (i+1)(j+1) mod 2^32; b[255][255] = 0 and
    b[127][255] = 2^31 (= INT32_MIN) -- the wrap pins of SURVEY 8.2.5 at a size
    a CPU test can afford."""
    n, m = 256, 300
    a = np.full((n, m), 1 << 16, dtype=np.int32)
    i = np.arange(n, dtype=np.int64)[:, None] + 1
    j = np.arange(m, dtype=np.int64)[None, :] + 1
    ref = ((1 << 16) * i * j) % (1 << 32)
    for form in FORMS:
        got = form(a).view(np.uint32).astype(np.int64)
        assert np.array_equal(got, ref)
    b = oracle.sat(a)
    assert b[255, 255] == 0
    assert b[127, 255] == np.int32(-2**31)


@pytest.mark.parametrize("n,m", [(17, 29), (29, 17), (64, 5)])
def test_separable_closed_form(n, m):
    """a[i][j] = f(i) g(j) => b[i][j] = F(i) G(j), F,G = 1-D cumsums; f != g
    so a transposed operand fails."""
    f = (np.arange(n, dtype=np.int64) * 3 + 1)
    g = (np.arange(m, dtype=np.int64) % 7 + 2)
    a = (f[:, None] * g[None, :]).astype(np.int32)
    ref = np.cumsum(f)[:, None] * np.cumsum(g)[None, :]
    for form in FORMS:
        assert np.array_equal(form(a).astype(np.int64), ref)
        assert np.array_equal(form(a.astype(np.float32)), ref.astype(np.float64))


# ---------------------------------------------------------------- special cases
@pytest.mark.parametrize("shape", [(1, 777), (777, 1)])
def test_1d_is_cumsum(shape):
    rng = np.random.default_rng(5)
    a = rng.integers(-2**31, 2**31, size=shape, dtype=np.int64).astype(np.int32)
    ref = np.cumsum(a.view(np.uint32).astype(np.uint64).ravel()) % (1 << 32)
    for form in FORMS:
        assert np.array_equal(form(a).view(np.uint32).ravel().astype(np.uint64), ref)
    af = rng.random(shape).astype(np.float32)
    reff = np.cumsum(af.astype(np.float64).ravel())
    for form in FORMS:
        assert np.allclose(form(af).ravel(), reff, rtol=1e-15, atol=0)


def test_empty():
    for shape in [(0, 5), (5, 0), (0, 0)]:
        a = np.zeros(shape, dtype=np.int32)
        assert oracle.sat(a).shape == shape


# ---------------------------------------------------------------- invariants
def test_inclusion_exclusion_recovers_input():
    """a = Delta_i Delta_j b exactly mod 2^32."""
    a = make_np(67, 131, "int32", "u32", seed=9)
    b = oracle.sat(a).view(np.uint32)
    pad = np.zeros((68, 132), dtype=np.uint32)
    pad[1:, 1:] = b
    with np.errstate(over="ignore"):
        rec = pad[1:, 1:] - pad[:-1, 1:] - pad[1:, :-1] + pad[:-1, :-1]
    assert np.array_equal(rec, a.view(np.uint32))


def test_transpose_and_linearity():
    a = make_np(23, 41, "int32", "u32", seed=1)
    c = make_np(23, 41, "int32", "u32", seed=2)
    assert np.array_equal(oracle.sat(np.ascontiguousarray(a.T)), oracle.sat(a).T)
    with np.errstate(over="ignore"):
        s = (a.view(np.uint32) + c.view(np.uint32)).view(np.int32)
        lhs = oracle.sat(s).view(np.uint32)
        rhs = oracle.sat(a).view(np.uint32) + oracle.sat(c).view(np.uint32)
    assert np.array_equal(lhs, rhs)


def test_formulations_agree_u32():
    a = make_np(200, 333, "int32", "u32", seed=4)
    r = oracle.sat(a)
    assert np.array_equal(oracle.sat_eq1(a), r)
    assert np.array_equal(oracle.sat_2pass(a), r)


def test_float64_exact_on_dyadic():
    """Inputs k 2^-24 make every float64 partial sum exact: the
    oracle must equal integer arithmetic on k exactly."""
    a = make_np(150, 97, "float32", "unit", seed=8)
    k = (a.astype(np.float64) * 2.0**24).astype(np.int64)
    assert np.array_equal(k.astype(np.float64) * 2.0**-24, a.astype(np.float64))
    ref = np.cumsum(np.cumsum(k, axis=0), axis=1).astype(np.float64) * 2.0**-24
    for form in FORMS:
        assert np.array_equal(form(a), ref)


def test_stream_strips_equal_full():
    a = make_np(100, 57, "int32", "u32", seed=6)
    full = oracle.sat(a)
    st = oracle.Stream(57, True)
    parts = [st.feed(a[s:e]) for s, e in [(0, 13), (13, 14), (14, 60), (60, 100)]]
    assert np.array_equal(np.concatenate(parts), full)
    # Formula (1) continued from the previous strip's last SAT row
    assert np.array_equal(oracle.sat_eq1(a[40:], prev_row=full[39]), full[40:])


def test_sat_at_matches():
    a = make_np(31, 45, "float32", "unit", seed=2)
    b = oracle.sat(a)
    for (i, j) in [(0, 0), (30, 44), (7, 19), (30, 0), (0, 44)]:
        assert oracle.sat_at(a, i, j) == b[i, j]
    ai = make_np(31, 45, "int32", "u32", seed=2)
    bi = oracle.sat(ai)
    for (i, j) in [(0, 0), (30, 44), (7, 19)]:
        assert oracle.sat_at(ai, i, j) == bi[i, j]


def test_sharding_invariant():
    """Strip p's SAT = local SAT + row prefix of carry_p (the exclusive rank
    scan of column totals), bit-exact mod 2^32."""
    a = make_np(64, 48, "int32", "u32", seed=12)
    full = oracle.sat(a).view(np.uint32)
    bounds = [0, 10, 11, 40, 64]
    P = len(bounds) - 1
    totals = np.stack([oracle.column_totals(a[bounds[p]:bounds[p + 1]]) for p in range(P)])
    # the bottom-row differences of a strip SAT are its column totals
    loc0 = oracle.sat(a[0:10]).view(np.uint32)
    with np.errstate(over="ignore"):
        assert np.array_equal(np.diff(np.concatenate([[0], loc0[-1]]).astype(np.uint32)),
                              totals[0].view(np.uint32))
    for p in range(P):
        carry = oracle.rank_exscan(totals, p).view(np.uint32)
        assert np.array_equal(carry, a[:bounds[p]].view(np.uint32).sum(axis=0, dtype=np.uint64).astype(np.uint32))
        loc = oracle.sat(a[bounds[p]:bounds[p + 1]]).view(np.uint32)
        with np.errstate(over="ignore"):
            top = np.cumsum(carry.astype(np.uint64)).astype(np.uint32)
            assert np.array_equal(loc + top[None, :], full[bounds[p]:bounds[p + 1]])


def test_max_rel_err():
    assert oracle.max_rel_err(np.array([1.0, 2.0]), np.array([1.0, 2.0])) == 0.0
    assert abs(oracle.max_rel_err(np.array([1.0, 2.2]), np.array([1.0, 2.0])) - 0.1) < 1e-12


# ---------------------------------------------------------------- float64 input
# The paper computes in double.  Pins for the d64 family.
@pytest.mark.parametrize("form", FORMS + [oracle.sat_brute])
def test_fig3_float64(fig3, form):
    a, cp, b = fig3
    got = form(a.astype(np.float64))
    assert got.dtype == np.float64 and np.array_equal(got, b.astype(np.float64))


@pytest.mark.parametrize("n,m", [(1, 1), (2, 7), (7, 2), (9, 13)])
def test_brute_small_float64(n, m):
    """Pure-Python double sum of exact dyadic values (no oracle code)."""
    a = make_np(n, m, "float64", "unit", seed=n * 31 + m)
    ref = np.array(py_brute(a.tolist()), dtype=np.float64)
    for form in FORMS + [oracle.sat_brute]:
        assert np.array_equal(form(a), ref)


def test_float64_dyadic_exact():
    """float64 "unit" inputs are k 2^-24: every partial sum below 2^29 is exact,
    so each formulation equals integer arithmetic on k exactly."""
    a = make_np(211, 173, "float64", "unit", seed=12)
    k = (a * 2.0**24).astype(np.int64)
    assert np.array_equal(k.astype(np.float64) * 2.0**-24, a)
    ref = np.cumsum(np.cumsum(k, axis=0), axis=1).astype(np.float64) * 2.0**-24
    for form in FORMS:
        assert np.array_equal(form(a), ref)
    # inclusion-exclusion recovers the input exactly (all values exact)
    b = oracle.sat(a)
    pad = np.zeros((212, 174))
    pad[1:, 1:] = b
    assert np.array_equal(pad[1:, 1:] - pad[:-1, 1:] - pad[1:, :-1] + pad[:-1, :-1], a)


def test_float64_unit53_vs_exact_rationals():
    """Full-mantissa inputs: the float64 oracle is within the recursive-summation
    bound (i + j + 2) u b[i][j] of the exact rational SAT (fractions)."""
    from fractions import Fraction
    a = make_np(12, 17, "float64", "unit53", seed=3)
    fa = [[Fraction(x) for x in row] for row in a.tolist()]
    exact = py_brute(fa)
    u = 2.0 ** -53
    for form in FORMS:
        got = form(a)
        for i in range(12):
            for j in range(17):
                err = abs(Fraction(got[i, j]) - exact[i][j])
                assert err <= (i + j + 2) * u * exact[i][j] * Fraction(101, 100)


@pytest.mark.parametrize("n,m", [(17, 29), (29, 17)])
def test_separable_closed_form_float64(n, m):
    f = (np.arange(n, dtype=np.int64) * 5 + 2)
    g = (np.arange(m, dtype=np.int64) % 11 + 1)
    a = (f[:, None] * g[None, :]).astype(np.float64)
    ref = (np.cumsum(f)[:, None] * np.cumsum(g)[None, :]).astype(np.float64)
    for form in FORMS:
        assert np.array_equal(form(a), ref)


@pytest.mark.parametrize("shape", [(1, 999), (999, 1)])
def test_1d_is_cumsum_float64(shape):
    """One row / one column: both are sequential left-to-right sums, bit-equal
    to numpy's cumsum (a library routine)."""
    a = make_np(*shape, "float64", "unit53", seed=4)
    for form in FORMS:
        assert np.array_equal(form(a).ravel(), np.cumsum(a.ravel()))


# ---------------------------------------------------------------- box filter
def py_box(a, rr, rc):
    """Pure-Python windowed sum (independent of the oracle's C code)."""
    n, m = len(a), len(a[0])
    return [[sum(a[k][l] for k in range(max(0, i - rr), min(n - 1, i + rr) + 1)
                 for l in range(max(0, j - rc), min(m - 1, j + rc) + 1))
             for j in range(m)] for i in range(n)]


@pytest.mark.parametrize("n,m,rr,rc", [(1, 1, 0, 0), (3, 4, 1, 1), (5, 7, 2, 1), (7, 5, 0, 3),
                                       (6, 6, 9, 9), (9, 13, 1, 4)])
def test_box_brute(n, m, rr, rc):
    a = make_np(n, m, "int32", "u8", seed=n * m)
    assert np.array_equal(oracle.box_filter(a, rr, rc), np.array(py_box(a.tolist(), rr, rc)))
    f = make_np(n, m, "float64", "unit", seed=n + m)
    assert np.array_equal(oracle.box_filter(f, rr, rc), np.array(py_box(f.tolist(), rr, rc)))


def test_box_worked_3x4():
    a = np.arange(12, dtype=np.int32).reshape(3, 4)
    assert oracle.box_filter(a, 1, 1).tolist() == [[10, 18, 24, 18], [27, 45, 54, 39],
                                                   [26, 42, 48, 34]]


def test_box_closed_forms():
    n, m, rr, rc = 37, 53, 3, 5
    ones = np.ones((n, m), dtype=np.int32)
    i, j = np.arange(n), np.arange(m)
    ci = np.minimum(n - 1, i + rr) - np.maximum(0, i - rr) + 1
    cj = np.minimum(m - 1, j + rc) - np.maximum(0, j - rc) + 1
    assert np.array_equal(oracle.box_filter(ones, rr, rc), ci[:, None] * cj[None, :])
    # separable a = f(i) g(j): window sums factor (f != g catches a swap of rr/rc)
    f = np.arange(n, dtype=np.int64) % 5 + 1
    g = np.arange(m, dtype=np.int64) % 3 + 2
    a = (f[:, None] * g[None, :]).astype(np.int32)
    wf = np.array([f[max(0, k - rr):k + rr + 1].sum() for k in range(n)])
    wg = np.array([g[max(0, k - rc):k + rc + 1].sum() for k in range(m)])
    assert np.array_equal(oracle.box_filter(a, rr, rc), wf[:, None] * wg[None, :])
    # radius 0 is the identity; a radius covering everything is the total
    b = make_np(20, 30, "int32", "u32", seed=3)
    assert np.array_equal(oracle.box_filter(b, 0, 0), b)
    tot = b.view(np.uint32).sum(dtype=np.uint64) % 2**32
    assert (oracle.box_filter(b, 40, 40).view(np.uint32) == tot).all()
    # the box mean of a constant is the constant
    c = np.full((9, 11), 0.75, dtype=np.float32)
    assert np.allclose(oracle.box_filter(c, 2, 3, normalize=True), 0.75, rtol=0, atol=1e-15)


def test_box_equals_four_sat_reads():
    """Inclusion-exclusion over the oracle SAT equals the direct
    windowed sum: the same quantity two ways."""
    a = make_np(40, 50, "int32", "u32", seed=11)
    b = oracle.sat(a)
    box = oracle.box_filter(a, 2, 3)
    for (i, j) in [(0, 0), (39, 49), (10, 3), (2, 47), (20, 25)]:
        r0, r1, c0, c1 = max(0, i - 2), min(39, i + 2), max(0, j - 3), min(49, j + 3)
        assert np.uint32(oracle.rect_sum(b, r0, c0, r1, c1)) == box.view(np.uint32)[i, j]
