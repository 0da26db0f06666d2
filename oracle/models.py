"""Step-by-step CPU models of the paper's SAT algorithms -- TEST INFRASTRUCTURE.

These follow Kasagi, Nakano, Ito (ICPP 2014, /root/reference/PAPER.md) in the
paper's own order and notation, block by block, so that the worked examples of
Figs. 8-11 can be checked value by value and the carry algebra of the B200
look-back can be related to the paper's.  They are slow
numpy/pure-Python code for tiny inputs; they are NOT the oracle's definition
(that is ``oracle.sat``) and the product path never imports them.

Notation: ``w`` = block side (the paper's w = number of banks);
B(I,J) = the w x w block in block-row I, block-column J.
Matrices may be rectangular here (rows, cols multiples of w), the paper's are
square (reading R2).  Arithmetic is done in the input's numpy dtype (int64 for
the figures, uint32 for wrap tests, float64 for floats).
"""
from __future__ import annotations

import numpy as np


def _cum(x, axis):
    return np.cumsum(x, axis=axis, dtype=x.dtype)


def block_sat(x: np.ndarray) -> np.ndarray:
    """SAT of one block: column-wise then row-wise prefix sums."""
    return _cum(_cum(x, 0), 1)


# ---------------------------------------------------------------------------
# Formula (1) / 4R1W on anti-diagonals (Sec. VI, Fig. 10)
# ---------------------------------------------------------------------------
def four_r_one_w(a: np.ndarray):
    """4R1W: Stage t computes b[i][j] for all i + j = t by Formula (1),
    b[i][j] = a[i][j] + b[i-1][j] + b[i][j-1] - b[i-1][j-1] (out-of-range terms 0).

    Returns (b, stages) where stages[t] = list of (i, j, b[i][j]) in order of i.
    """
    n, m = a.shape
    b = np.zeros_like(a)
    stages = []
    for t in range(n + m - 1):
        diag = []
        for i in range(max(0, t - m + 1), min(n, t + 1)):
            j = t - i
            v = a[i, j]
            if i > 0:
                v = v + b[i - 1, j]
            if j > 0:
                v = v + b[i, j - 1]
            if i > 0 and j > 0:
                v = v - b[i - 1, j - 1]
            b[i, j] = v
            diag.append((i, j, v))
        stages.append(diag)
    return b, stages


# ---------------------------------------------------------------------------
# 2R1W (Sec. V, Figs. 8 and 9)
# ---------------------------------------------------------------------------
def two_r_one_w(a: np.ndarray, w: int, counters: dict | None = None):
    """2R1W SAT, following Steps 1, 2, 3-1, 3-2 of P:L1059-L1137.

    Step 1: per block, column-wise sums C, row-wise sums R and block sum S
            (bottom blocks' column sums and right blocks' row sums are not
            needed).
    Step 2: column-wise prefix-sums of C, row-wise prefix-sums of R, SAT of S
            (computed directly here: reading R11, no recursion).
    Step 3-1: add the C, R and S carries to the block's top row, leftmost
            column and top-left corner.
    Step 3-2: SAT of the modified block.

    Returns (b, info) with the intermediates used by Figs. 8 and 9.
    ``counters`` (optional) accumulates element reads/writes of a and b.
    """
    n, m = a.shape
    assert n % w == 0 and m % w == 0, "model handles whole blocks (reading R2)"
    NI, NJ = n // w, m // w
    # Step 1
    C = np.zeros((NI, m), dtype=a.dtype)        # column-wise sums per block-row
    R = np.zeros((n, NJ), dtype=a.dtype)        # row-wise sums per block-column
    S = np.zeros((NI, NJ), dtype=a.dtype)
    for I in range(NI):
        for J in range(NJ):
            blk = a[I * w:(I + 1) * w, J * w:(J + 1) * w]
            C[I, J * w:(J + 1) * w] = blk.sum(axis=0, dtype=a.dtype)
            R[I * w:(I + 1) * w, J] = blk.sum(axis=1, dtype=a.dtype)
            S[I, J] = blk.sum(dtype=a.dtype)
    if counters is not None:
        counters["read"] = counters.get("read", 0) + a.size
    # Step 2 (only the first NI-1 / NJ-1 block rows / columns are ever used)
    Cp = _cum(C[:NI - 1], 0)
    Rp = _cum(R[:, :NJ - 1], 1)
    SS = block_sat(S[:NI - 1, :NJ - 1])
    # Step 3-1 and 3-2
    b = np.zeros_like(a)
    after31 = {}
    for I in range(NI):
        for J in range(NJ):
            x = a[I * w:(I + 1) * w, J * w:(J + 1) * w].copy()
            if I > 0:
                x[0, :] += Cp[I - 1, J * w:(J + 1) * w]
            if J > 0:
                x[:, 0] += Rp[I * w:(I + 1) * w, J - 1]
            if I > 0 and J > 0:
                x[0, 0] += SS[I - 1, J - 1]
            after31[(I, J)] = x.copy()
            b[I * w:(I + 1) * w, J * w:(J + 1) * w] = block_sat(x)
    if counters is not None:
        counters["read"] += a.size
        counters["write"] = counters.get("write", 0) + a.size
    info = dict(C=C, R=R, S=S, C_prefix=Cp, R_prefix=Rp, SAT_S=SS, after_3_1=after31)
    return b, info


# ---------------------------------------------------------------------------
# 1R1W (Sec. VI, Fig. 11): block-wise 4R1W, carries recovered
# from neighbours' final SAT values by pairwise subtraction.
# ---------------------------------------------------------------------------
def _carries_from_neighbours(b, I, J, w):
    """C, R, S for B(I,J) from already-final SAT values.

    C[c] = b[r0-1][c] - b[r0-1][c-1]   (bottom row of B(I-1,J), the corner of
                                        B(I-1,J-1) for the first column)
    R[r] = b[r][c0-1] - b[r-1][c0-1]   (right column of B(I,J-1), same corner)
    S    = b[r0-1][c0-1]               (bottom-right corner of B(I-1,J-1))
    Out-of-range SAT values are 0.  Also returns how many b values were read.
    """
    r0, c0 = I * w, J * w
    z = b.dtype.type(0)

    def bv(i, j):
        return b[i, j] if (i >= 0 and j >= 0) else z
    C = np.array([bv(r0 - 1, c) - bv(r0 - 1, c - 1) for c in range(c0, c0 + w)], dtype=b.dtype)
    R = np.array([bv(r, c0 - 1) - bv(r - 1, c0 - 1) for r in range(r0, r0 + w)], dtype=b.dtype)
    S = bv(r0 - 1, c0 - 1)
    reads = (w if I > 0 else 0) + (w if J > 0 else 0) + (1 if (I > 0 and J > 0) else 0)
    return C, R, S, reads


def _apply_block(a, b, I, J, w, C, R, S):
    """Step 3-1 (add carries) and Step 3-2 (block SAT) of 2R1W."""
    x = a[I * w:(I + 1) * w, J * w:(J + 1) * w].copy()
    x[0, :] += C
    x[:, 0] += R
    x[0, 0] += S
    b[I * w:(I + 1) * w, J * w:(J + 1) * w] = block_sat(x)
    return x


def one_r_one_w(a: np.ndarray, w: int, counters: dict | None = None):
    """1R1W: Stage t (t = 0 .. NI+NJ-2) computes every B(I,J) with I + J = t.

    Returns (b, info) with info["carries"][(I,J)] = (C, R, S), the stage list
    and info["after_3_1"].
    """
    with np.errstate(over="ignore"):
        n, m = a.shape
        assert n % w == 0 and m % w == 0
        NI, NJ = n // w, m // w
        b = np.zeros_like(a)
        carries, after31, stages = {}, {}, []
        for t in range(NI + NJ - 1):
            blocks = [(I, t - I) for I in range(max(0, t - NJ + 1), min(NI, t + 1))]
            stages.append(blocks)
            for (I, J) in blocks:
                C, R, S, reads = _carries_from_neighbours(b, I, J, w)
                carries[(I, J)] = (C, R, S)
                after31[(I, J)] = _apply_block(a, b, I, J, w, C, R, S)
                if counters is not None:
                    counters["read"] = counters.get("read", 0) + w * w
                    counters["edge_read"] = counters.get("edge_read", 0) + reads
                    counters["write"] = counters.get("write", 0) + w * w
        return b, dict(carries=carries, after_3_1=after31, stages=stages)


# ---------------------------------------------------------------------------
# (1+r)R1W (Sec. VII, Fig. 12)
# ---------------------------------------------------------------------------
def region_split(NI: int, NJ: int, t_A: int):
    """Blocks of (A) top-left triangle I+J < t_A, (B) bottom-right triangle
    I+J > NI+NJ-2-t_A, (C) the rest (reading R10: triangles bounded by block
    anti-diagonals).  Returns dict name -> set of (I,J)."""
    last = NI + NJ - 2
    A, B, Cr = set(), set(), set()
    for I in range(NI):
        for J in range(NJ):
            t = I + J
            if t < t_A:
                A.add((I, J))
            elif t > last - t_A:
                B.add((I, J))
            else:
                Cr.add((I, J))
    return dict(A=A, B=B, C=Cr)


def r_effective(NI: int, NJ: int, t_A: int) -> float:
    """Fraction r of blocks done by 2R1W (A and B together cover ~ r n^2)."""
    s = region_split(NI, NJ, t_A)
    return (len(s["A"]) + len(s["B"])) / float(NI * NJ)


def one_plus_r_r_one_w(a: np.ndarray, w: int, t_A: int, counters: dict | None = None):
    """(1+r)R1W: 2R1W on (A), then 1R1W on (C), then 2R1W on (B).

    2R1W on a region (reading R10): Step 1 reduces every region block; Step 2
    forms the carries from the column/row sums of region blocks above/left,
    starting from the final SAT values on the region's boundary (pairwise
    subtraction, as 1R1W does); Steps 3-1/3-2 as in 2R1W.
    For (A) the boundary is the matrix edge, so this is exactly 2R1W.
    """
    with np.errstate(over="ignore"):
        n, m = a.shape
        NI, NJ = n // w, m // w
        reg = region_split(NI, NJ, t_A)
        b = np.zeros_like(a)
        z = a.dtype.type(0)

        def bv(i, j):
            return b[i, j] if (i >= 0 and j >= 0) else z

        def two_r_one_w_region(blocks):
            # Step 1: column sums / row sums / sums of every block of the region.
            Cs, Rs, Ss = {}, {}, {}
            for (I, J) in blocks:
                blk = a[I * w:(I + 1) * w, J * w:(J + 1) * w]
                Cs[(I, J)] = blk.sum(axis=0, dtype=a.dtype)
                Rs[(I, J)] = blk.sum(axis=1, dtype=a.dtype)
                Ss[(I, J)] = blk.sum(dtype=a.dtype)
            if counters is not None:
                counters["read"] = counters.get("read", 0) + w * w * len(blocks)
            # Step 2: carries.  The first region block of a column (row) starts
            # from the boundary SAT values by pairwise subtraction.
            for (I, J) in sorted(blocks):
                r0, c0 = I * w, J * w
                # column carries: walk up through region blocks to the boundary
                Cc = np.zeros(w, dtype=a.dtype)
                k = I - 1
                while k >= 0 and (k, J) in blocks:
                    Cc = Cc + Cs[(k, J)]
                    k -= 1
                rb = (k + 1) * w - 1        # boundary row (last non-region row)
                Cc = Cc + np.array([bv(rb, c) - bv(rb, c - 1) for c in range(c0, c0 + w)],
                                   dtype=a.dtype)
                Rc = np.zeros(w, dtype=a.dtype)
                k = J - 1
                while k >= 0 and (I, k) in blocks:
                    Rc = Rc + Rs[(I, k)]
                    k -= 1
                cb = (k + 1) * w - 1
                Rc = Rc + np.array([bv(r, cb) - bv(r - 1, cb) for r in range(r0, r0 + w)],
                                   dtype=a.dtype)
                # corner = sum of everything above-left: boundary SAT value
                # at (r0-1, c0-1) is final unless that block is in the region.
                Sc = _corner(I, J, blocks, Ss, Cs, Rs, bv, w, a.dtype)
                _apply_block(a, b, I, J, w, Cc, Rc, Sc)
            if counters is not None:
                counters["read"] += w * w * len(blocks)
                counters["write"] = counters.get("write", 0) + w * w * len(blocks)

        two_r_one_w_region(reg["A"])
        # 1R1W on (C), stage by stage
        for t in range(NI + NJ - 1):
            for I in range(max(0, t - NJ + 1), min(NI, t + 1)):
                J = t - I
                if (I, J) in reg["C"]:
                    C, R, S, _ = _carries_from_neighbours(b, I, J, w)
                    _apply_block(a, b, I, J, w, C, R, S)
                    if counters is not None:
                        counters["read"] = counters.get("read", 0) + w * w
                        counters["write"] = counters.get("write", 0) + w * w
        two_r_one_w_region(reg["B"])
        return b, dict(regions=reg, r=r_effective(NI, NJ, t_A))


def _corner(I, J, blocks, Ss, Cs, Rs, bv, w, dt):
    """sum_{k < r0, l < c0} a[k][l] for region block (I,J).

    Walk up-left: the value b[r0-1][c0-1] is final when B(I-1,J-1) is outside
    the region; otherwise it is the corner of B(I-1,J-1) plus that block's own
    sum plus the column/row sums of region blocks between -- computed here by
    summing the region's block sums S over the rectangle (I' < I, J' < J)
    restricted to the region, plus the boundary SAT value below-right of it.
    """
    r0, c0 = I * w, J * w
    if I == 0 or J == 0:
        return dt.type(0)
    if (I - 1, J - 1) not in blocks:
        return bv(r0 - 1, c0 - 1)
    # (A) and (B) are staircase triangles: region blocks above-left of (I,J)
    # form a staircase whose complement above-left is final in b.  Sum the
    # region blocks inside [0,I) x [0,J) and add the final SAT of the rest by
    # inclusion-exclusion over the staircase boundary.
    total = dt.type(0)
    for (i2, j2) in blocks:
        if i2 < I and j2 < J:
            total = total + Ss[(i2, j2)]
    # Non-region part of the rectangle [0, r0) x [0, c0): rows of each block
    # column j2 < J that lie above the first region block of that column.
    for j2 in range(J):
        k = I - 1
        while k >= 0 and (k, j2) in blocks:
            k -= 1
        rb = (k + 1) * w - 1   # last non-region row in this block column
        if rb >= 0:
            # sum of a[0..rb][j2*w .. j2*w+w-1] = SAT differences
            total = total + (bv(rb, (j2 + 1) * w - 1) - bv(rb, j2 * w - 1))
    return total
