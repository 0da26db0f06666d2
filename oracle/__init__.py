"""CPU oracle for the summed area table (SAT) -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product path
(``paper_conf_icpp_kasagini14_b200``) never imports it; the two share no code.

Definition followed (Kasagi, Nakano, Ito, ICPP 2014 -- /root/reference/PAPER.md):
  * P:L187-L193 (Sec. I, Fig. 3): ``b[i][j] = sum_{k<=i, l<=j} a[k][l]``,
    inclusive, obtainable as column-wise prefix-sums then row-wise prefix-sums.
  * P:L193 / P:L221: any rectangle sum is four SAT reads (inclusion-exclusion).
  * P:L1891-L1905 Formula (1); P:L2423-L2465 the 2R2W(CPU) and 4R1W(CPU)
    sequential baselines.

Element types (reading R3): int32 input is summed in uint32 (wraps
mod 2^32); float32 input is summed in float64; float64 input (the paper's own
precision) is summed in float64.  The heavy loops are plain C
(``sat_oracle.c``, single-threaded, gcc -O2) loaded with ctypes; small helpers
are numpy.  Every pin lives in ``tests/test_oracle.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sat_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

_P = ctypes.c_void_p
_I64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile ``sat_oracle.c`` into ``liboracle.so`` (gcc -O2, no -ffast-math)."""
    if force or not os.path.exists(_LIB_PATH) or (
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC)):
        tmp = _LIB_PATH + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        for k in _KINDS:
            getattr(lib, f"oracle_sat_{k}").argtypes = [_P, _P, _I64, _I64, _P]
            getattr(lib, f"oracle_sat_{k}_eq1").argtypes = [_P, _P, _I64, _I64, _P]
            getattr(lib, f"oracle_sat_{k}_2pass").argtypes = [_P, _P, _I64, _I64]
            getattr(lib, f"oracle_sat_{k}_brute").argtypes = [_P, _P, _I64, _I64]
            getattr(lib, f"oracle_sat_{k}_at").argtypes = [_P, _I64, _I64, _I64, _I64]
        for k in _KINDS:
            getattr(lib, f"oracle_box_{k}").argtypes = [_P, _P, _I64, _I64, _I64, _I64]
        lib.oracle_sat_u32_at.restype = ctypes.c_uint32
        lib.oracle_sat_f64_at.restype = ctypes.c_double
        lib.oracle_sat_d64_at.restype = ctypes.c_double
        _lib = lib
    return _lib


# C function families by input kind: u32 (int32/uint32 input, uint32 sums),
# f64 (float32 input, float64 sums), d64 (float64 input, float64 sums)
_KINDS = ("u32", "f64", "d64")


def _kind(a: np.ndarray) -> str:
    if a.dtype in (np.int32, np.uint32):
        return "u32"
    if a.dtype == np.float32:
        return "f64"
    if a.dtype == np.float64:
        return "d64"
    raise TypeError(f"oracle supports int32/uint32/float32/float64 inputs, got {a.dtype}")


def _prep(a: np.ndarray):
    """Return (contiguous input, is_int, output dtype)."""
    a = np.ascontiguousarray(a)
    if a.ndim != 2:
        raise ValueError("oracle expects a 2-D matrix")
    k = _kind(a)
    if k == "u32":
        return a.view(np.uint32), True, np.uint32
    return a, False, np.float64


def _fn(lib, a: np.ndarray, suffix: str = ""):
    return getattr(lib, f"oracle_sat_{_kind(a)}{suffix}")


def _ptr(x: np.ndarray):
    return x.ctypes.data_as(ctypes.c_void_p)


def _ret(out: np.ndarray, a_dtype) -> np.ndarray:
    return out.view(np.int32) if a_dtype == np.int32 else out


class Stream:
    """Streaming oracle state: feed consecutive row strips of one matrix.

    Keeps the running column sums ``colsum[j] = sum_{k<i} a[k][j]`` between
    strips (column-wise prefix-sums, then row-wise prefix-sums).
    """

    def __init__(self, cols: int, is_int: bool):
        self.cols = int(cols)
        self.is_int = bool(is_int)
        self.colsum = np.zeros(self.cols, dtype=np.uint32 if is_int else np.float64)

    def feed(self, strip: np.ndarray) -> np.ndarray:
        a, is_int, odt = _prep(strip)
        if is_int != self.is_int or a.shape[1] != self.cols:
            raise ValueError("strip does not match stream")
        out = np.empty(a.shape, dtype=odt)
        lib = _load()
        fn = _fn(lib, a)
        if a.size:
            fn(_ptr(a), _ptr(out), a.shape[0], a.shape[1], _ptr(self.colsum))
        return _ret(out, strip.dtype)


def sat(a: np.ndarray) -> np.ndarray:
    """SAT by column-wise then row-wise prefix sums (row-fused, streaming C)."""
    a_c, is_int, _ = _prep(a)
    return Stream(a_c.shape[1], is_int).feed(a)


def sat_eq1(a: np.ndarray, prev_row: np.ndarray | None = None) -> np.ndarray:
    """SAT by Formula (1) in raster order (the paper's 4R1W(CPU))."""
    a_c, is_int, odt = _prep(a)
    out = np.empty(a_c.shape, dtype=odt)
    lib = _load()
    fn = _fn(lib, a_c, "_eq1")
    pr = None
    if prev_row is not None:
        pr = np.ascontiguousarray(prev_row)
        pr = pr.view(np.uint32) if is_int else np.ascontiguousarray(pr, dtype=np.float64)
    if a_c.size:
        fn(_ptr(a_c), _ptr(out), a_c.shape[0], a_c.shape[1],
           _ptr(pr) if pr is not None else None)
    return _ret(out, a.dtype)


def sat_2pass(a: np.ndarray) -> np.ndarray:
    """SAT by the paper's 2R2W(CPU): whole column pass, then whole row pass."""
    a_c, is_int, odt = _prep(a)
    out = np.empty(a_c.shape, dtype=odt)
    lib = _load()
    fn = _fn(lib, a_c, "_2pass")
    if a_c.size:
        fn(_ptr(a_c), _ptr(out), a_c.shape[0], a_c.shape[1])
    return _ret(out, a.dtype)


def sat_brute(a: np.ndarray) -> np.ndarray:
    """SAT by the double sum written out (O(n^2 m^2)); tiny inputs only."""
    a_c, is_int, odt = _prep(a)
    if a_c.size > 1 << 16:
        raise ValueError("sat_brute is for tiny inputs")
    out = np.empty(a_c.shape, dtype=odt)
    lib = _load()
    fn = _fn(lib, a_c, "_brute")
    if a_c.size:
        fn(_ptr(a_c), _ptr(out), a_c.shape[0], a_c.shape[1])
    return _ret(out, a.dtype)


def sat_at(a: np.ndarray, i: int, j: int):
    """One element b[i][j] = sum_{k<=i, l<=j} a[k][l] (sampled parity)."""
    a_c, is_int, _ = _prep(a)
    lib = _load()
    if is_int:
        v = lib.oracle_sat_u32_at(_ptr(a_c), a_c.shape[0], a_c.shape[1], int(i), int(j))
        return np.uint32(v).view(np.int32) if a.dtype == np.int32 else np.uint32(v)
    return float(_fn(lib, a_c, "_at")(_ptr(a_c), a_c.shape[0], a_c.shape[1], int(i), int(j)))


def rect_sum(b: np.ndarray, r0: int, c0: int, r1: int, c1: int):
    """Sum of a[r0..r1][c0..c1] (inclusive) from four SAT reads.

    Integer SATs are combined in uint32 (mod 2^32); float SATs in float64.
    """
    bb = b.view(np.uint32) if b.dtype == np.int32 else b

    def at(i, j):
        if i < 0 or j < 0:
            return bb.dtype.type(0)
        return bb[i, j]
    with np.errstate(over="ignore"):
        return at(r1, c1) - at(r0 - 1, c1) - at(r1, c0 - 1) + at(r0 - 1, c0 - 1)


def box_filter(a: np.ndarray, rr: int, rc: int, normalize: bool = False) -> np.ndarray:
    """Box filter by its plain definition (the SAT's use case,
    P:L193, L221): out[i][j] = sum of a over rows |k - i| <= rr and columns
    |l - j| <= rc, clipped to the matrix.  int32 -> uint32 sums (returned as
    int32), float -> float64.  ``normalize`` divides by the clipped window's
    element count (a box mean; float inputs only).  O(n m rr rc): small inputs."""
    a_c, is_int, odt = _prep(a)
    out = np.empty(a_c.shape, dtype=odt)
    if a_c.size:
        getattr(_load(), f"oracle_box_{_kind(a_c)}")(_ptr(a_c), _ptr(out), a_c.shape[0],
                                                      a_c.shape[1], int(rr), int(rc))
    if normalize:
        if is_int:
            raise ValueError("normalize is for float inputs")
        n, m = a_c.shape
        i = np.arange(n)
        j = np.arange(m)
        ci = np.minimum(n - 1, i + rr) - np.maximum(0, i - rr) + 1
        cj = np.minimum(m - 1, j + rc) - np.maximum(0, j - rc) + 1
        out = out / (ci[:, None] * cj[None, :]).astype(np.float64)
    return _ret(out, a.dtype)


def column_totals(a: np.ndarray) -> np.ndarray:
    """Column sums of a strip (the sharded mode's exchanged vector).

    int32 -> uint32 (mod 2^32, returned as int32), float32/float64 -> float64.
    """
    a_c, is_int, _ = _prep(a)
    if is_int:
        return a_c.sum(axis=0, dtype=np.uint64).astype(np.uint32).view(np.int32)
    return a_c.astype(np.float64).sum(axis=0)


def rank_exscan(totals_by_rank: np.ndarray, rank: int) -> np.ndarray:
    """carry_p[j] = sum_{q<p} totals_q[j]: column sums of every row above strip p."""
    t = np.asarray(totals_by_rank)
    if t.dtype == np.int32:
        out = t[:rank].view(np.uint32).sum(axis=0, dtype=np.uint64).astype(np.uint32)
        return out.view(np.int32)
    return t[:rank].astype(np.float64).sum(axis=0)


def max_rel_err(gpu: np.ndarray, ref: np.ndarray) -> float:
    """max_ij |g - o| / max(|o|, 1e-30) (the north-star float32 metric)."""
    g = np.asarray(gpu, dtype=np.float64)
    o = np.asarray(ref, dtype=np.float64)
    if g.size == 0:
        return 0.0
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), 1e-30)))
