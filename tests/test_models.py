"""Pins for the step-by-step paper models (``oracle/models.py``): the worked
examples of Figs. 8, 9, 10, 11 (tile w = 3) and the read/write counts of
Lemma 4, Theorem 6 and Theorem 7.  CPU only."""
import numpy as np
import pytest

import oracle
from oracle import models
from conftest import load_keyed


def test_2r1w_fig3_and_fig8(fig3):
    a, _, b = fig3
    a = a.astype(np.int64)
    got, info = models.two_r_one_w(a, 3)
    assert np.array_equal(got, b)
    f8 = load_keyed("fig8_w3.txt")
    assert info["S"].ravel().tolist() == f8["S"]
    assert info["C"][0].tolist() == f8["C_row0"]
    assert info["C"][1].tolist() == f8["C_row1"]
    assert info["C_prefix"][1].tolist() == f8["C_prefix_row1"]
    assert info["SAT_S"].ravel().tolist() == f8["SAT_S_topleft"]


def test_2r1w_fig9_block21(fig3):
    a, _, b = fig3
    got, info = models.two_r_one_w(a.astype(np.int64), 3)
    f9 = load_keyed("fig9_block21.txt")
    assert a[6:9, 3:6].ravel().tolist() == f9["input"]
    # Step 3-1 carries of B(2,1): C prefix of block-row 1, R prefix of block-col 0, SAT(S)[1][0]
    assert info["C_prefix"][1, 3:6].tolist() == f9["C"]
    assert info["R_prefix"][6:9, 0].tolist() == f9["R"]
    assert int(info["SAT_S"][1, 0]) == f9["S"][0]
    assert info["after_3_1"][(2, 1)].ravel().tolist() == f9["after_3_1"]
    assert got[6:9, 3:6].ravel().tolist() == f9["after_3_2"]


def test_1r1w_fig11(fig3):
    a, _, b = fig3
    got, info = models.one_r_one_w(a.astype(np.int64), 3)
    assert np.array_equal(got, b)
    f9 = load_keyed("fig9_block21.txt")
    C, R, S = info["carries"][(2, 1)]
    assert C.tolist() == f9["C"] and R.tolist() == f9["R"] and int(S) == f9["S"][0]
    assert got[5, 3:6].tolist() == f9["fig11_bottom_row_B11"]
    assert got[6:9, 2].tolist() == f9["fig11_right_col_B20"]
    assert info["after_3_1"][(2, 1)].ravel().tolist() == f9["after_3_1"]
    # Stage 3 computes B(I,J) with I + J = 3 (Fig. 11); 2n/w - 1 = 5 stages.
    assert len(info["stages"]) == 5
    assert (2, 1) in info["stages"][3] and (1, 2) in info["stages"][3]


def test_4r1w_fig10(fig3):
    a, _, b = fig3
    got, stages = models.four_r_one_w(a.astype(np.int64))
    assert np.array_equal(got, b)
    f10 = load_keyed("fig10_stage7.txt")
    assert [int(a[i, j]) for (i, j, _) in stages[7]] == f10["input"]
    assert [int(v) for (_, _, v) in stages[7]] == f10["sat"]
    assert len(stages) == 2 * 9 - 1


@pytest.mark.parametrize("t_A", range(0, 6))
def test_1plusr_fig3(fig3, t_A):
    a, _, b = fig3
    got, info = models.one_plus_r_r_one_w(a.astype(np.int64), 3, t_A)
    assert np.array_equal(got, b)


@pytest.mark.parametrize("w,shape", [(3, (12, 15)), (4, (16, 8)), (2, (10, 14))])
def test_models_random_rect(w, shape):
    rng = np.random.default_rng(sum(shape) + w)
    a = rng.integers(0, 2**32, size=shape, dtype=np.uint64).astype(np.uint32)
    ref = oracle.sat(a.view(np.int32)).view(np.uint32)
    with np.errstate(over="ignore"):
        assert np.array_equal(models.two_r_one_w(a, w)[0], ref)
        assert np.array_equal(models.one_r_one_w(a, w)[0], ref)
        assert np.array_equal(models.four_r_one_w(a)[0], ref)
        NI, NJ = shape[0] // w, shape[1] // w
        for t_A in range(0, NI + NJ):
            assert np.array_equal(models.one_plus_r_r_one_w(a, w, t_A)[0], ref), t_A


def test_read_write_counts():
    """Lemma 4 / Theorem 6 / Theorem 7 (reconstructed): 2R1W reads
    each element twice, 1R1W once (+ at most 2w+1 edge values per block),
    (1+r)R1W (1+r) times; all write once."""
    w, n = 4, 32
    a = np.arange(n * n, dtype=np.int64).reshape(n, n) % 7
    c = {}
    models.two_r_one_w(a, w, c)
    assert c["read"] == 2 * n * n and c["write"] == n * n
    c = {}
    models.one_r_one_w(a, w, c)
    assert c["read"] == n * n and c["write"] == n * n
    assert c["edge_read"] <= (2 * w + 1) * (n // w) ** 2
    for t_A in (0, 2, 4):
        c = {}
        _, info = models.one_plus_r_r_one_w(a, w, t_A, c)
        r = info["r"]
        assert c["read"] == round((1 + r) * n * n) and c["write"] == n * n
    # reading R10: r_eff = t_A (t_A + 1) / (NI NJ) (two triangles of t_A(t_A+1)/2 blocks)
    assert abs(models.r_effective(8, 8, 4) - 20 / 64) < 1e-12
