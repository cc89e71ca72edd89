"""CPU ORACLE for the summed area table -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl reference``
legs may import this package.  The product (``paper_conf_ipps_emotofthni18_b200`` / libsat) never
imports it and shares no code with it.

Contents (PAPER.md cited as P:<line>; readings R<n> are listed in DESIGN.md):

* ``sat_u32`` / ``col_prefix_u32`` / ``row_prefix_u32`` -- the SAT as column-wise prefix sums then
  row-wise prefix sums (Fig. 2), uint32 wraparound (R1).  C: sat_oracle.c.
* ``sat_f32`` -- the same two passes in fp64 from fp32 input, plus absSAT = SAT(|a|) (R1, R10).
* ``Stream`` -- the streaming form (one row at a time; keeps the running column sums).
* ``region_sum`` -- S[U:D][L:R] of P:128-130.
* ``table2`` -- the per-tile sums LRS, LCS, LS, GRS, GCS, GS, GLS, GSAT of Table II (missing from
  the extracted text; reconstructed from their uses at P:144-150, P:162, P:192-243 -- R5),
  each written as the region sum that defines it.
* ``tile_order`` -- the diagonal-major serial numbering of Fig. 9 (R6).
* ``rect_sum`` -- the rectangle query of P:48; ``box_sum`` -- the box filter built from it.
* ``strip_carry_u32`` -- the carry row of a horizontal strip (column sums of all rows above it), read
  from the streaming state (R12, multi-GPU); ``Stream.colsums_f64`` is its fp64 counterpart.
* ``moments_f32`` -- the two SATs of a summed-area variance shadow map, SAT(a) and SAT(a*a) (P:50 and
  its ref. [8]), in fp64 from fp32 input, with their absSATs.
* ``f32_tolerance`` -- the fp32 acceptance bound of BASELINE.json north_star (R10).

Every function is pinned by tests/test_oracle.py against something other than itself (the test
named after each function is listed in DESIGN.md Sec. 3); none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
from pathlib import Path

import numpy as np

_HERE = Path(__file__).resolve().parent
_lib = None

_i64 = ctypes.c_int64
_vp = ctypes.c_void_p


def _load():
    global _lib
    if _lib is None:
        so = _HERE / "liboracle.so"
        if not so.exists() or so.stat().st_mtime < (_HERE / "sat_oracle.c").stat().st_mtime:
            import build_native  # repo root is on sys.path for tests / bench

            build_native.build_oracle()
        lib = ctypes.CDLL(str(so))
        for name in ("oracle_col_prefix_u32", "oracle_row_prefix_u32", "oracle_sat_u32"):
            getattr(lib, name).argtypes = [_vp, _vp, _i64, _i64, _i64]
            getattr(lib, name).restype = None
        lib.oracle_sat_f32_f64.argtypes = [_vp, _vp, _vp, _i64, _i64, _i64]
        lib.oracle_sat_f32_f64.restype = None
        lib.oracle_sat_f64.argtypes = [_vp, _vp, _i64, _i64]
        lib.oracle_sat_f64.restype = None
        lib.oracle_stream_new.argtypes = [_i64]
        lib.oracle_stream_new.restype = _vp
        lib.oracle_stream_free.argtypes = [_vp]
        lib.oracle_stream_free.restype = None
        lib.oracle_stream_colsums_u32.argtypes = [_vp, _vp]
        lib.oracle_stream_colsums_f64.argtypes = [_vp, _vp]
        lib.oracle_stream_rows_u32.argtypes = [_vp, _vp, _vp, _i64, _i64, _i64]
        lib.oracle_stream_rows_u32.restype = None
        lib.oracle_stream_rows_f32.argtypes = [_vp, _vp, _vp, _vp, _i64, _i64, _i64]
        lib.oracle_stream_rows_f32.restype = None
        lib.oracle_region_sum_u32.argtypes = [_vp, _i64, _i64, _i64, _i64, _i64]
        lib.oracle_region_sum_u32.restype = ctypes.c_uint32
        lib.oracle_region_sum_f64.argtypes = [_vp, _i64, _i64, _i64, _i64, _i64]
        lib.oracle_region_sum_f64.restype = ctypes.c_double
        _lib = lib
    return _lib


def _u32(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint32:
        return a
    if a.dtype.itemsize == 4 and a.dtype.kind in "iu":
        return a.view(np.uint32)
    return np.ascontiguousarray(a.astype(np.int64).astype(np.uint32))


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


# ------------------------------------------------------------------------------------ uint32 SAT
def col_prefix_u32(a: np.ndarray) -> np.ndarray:
    """Pass 1: column-wise prefix sums mod 2^32.  a: 2-D integer array."""
    a = _u32(a)
    c = np.empty_like(a)
    _load().oracle_col_prefix_u32(_ptr(a), _ptr(c), a.shape[0], a.shape[1], a.shape[1])
    return c


def row_prefix_u32(c: np.ndarray) -> np.ndarray:
    """Pass 2: row-wise prefix sums mod 2^32."""
    c = _u32(c)
    b = np.empty_like(c)
    _load().oracle_row_prefix_u32(_ptr(c), _ptr(b), c.shape[0], c.shape[1], c.shape[1])
    return b


def sat_u32(a: np.ndarray) -> np.ndarray:
    """SAT mod 2^32 of a 2-D int32/uint32 array (uint32 result; view as int32 for two's complement)."""
    a = _u32(a)
    b = np.empty_like(a)
    if a.size:
        _load().oracle_sat_u32(_ptr(a), _ptr(b), a.shape[0], a.shape[1], a.shape[1])
    return b


def sat_i32(a: np.ndarray) -> np.ndarray:
    return sat_u32(a).view(np.int32)


# ------------------------------------------------------------------------------------ fp64 SAT
def sat_f32(a: np.ndarray, with_abs: bool = True):
    """fp64 SAT (and fp64 absSAT) of a 2-D float32 array.  Returns (sat, abssat or None)."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    rows, cols = a.shape
    b = np.empty((rows, cols), dtype=np.float64)
    ab = np.empty((rows, cols), dtype=np.float64) if with_abs else None
    if a.size:
        _load().oracle_sat_f32_f64(_ptr(a), _ptr(b), _ptr(ab) if ab is not None else None, rows, cols, cols)
    return b, ab


def sat_f64(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.float64)
    b = np.empty_like(a)
    if a.size:
        _load().oracle_sat_f64(_ptr(a), _ptr(b), a.shape[0], a.shape[1])
    return b


def moments_f32(a: np.ndarray):
    """Summed-area variance shadow map moments (ref. [8] P:311): the SAT of a and the SAT of
    a*a, both by the column-then-row passes of P:46 in fp64 (a fp32 value squares exactly in fp64),
    each with its absSAT for the R10 tolerance.  Returns (sat1, abs1, sat2, abs2); abs2 == sat2."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    s1, ab1 = sat_f32(a)
    sq = a.astype(np.float64) * a.astype(np.float64)
    s2 = sat_f64(sq)
    return s1, ab1, s2, s2.copy()


# ------------------------------------------------------------------------------------ streaming
class Stream:
    """Streaming oracle: feed input rows top to bottom, get SAT rows back (O(cols) state)."""

    def __init__(self, cols: int):
        self.cols = cols
        self._s = _load().oracle_stream_new(cols)
        if not self._s:
            raise MemoryError("oracle_stream_new")
        self.row = 0

    def close(self):
        if self._s:
            _load().oracle_stream_free(self._s)
            self._s = None

    def __del__(self):  # pragma: no cover
        self.close()

    def rows_u32(self, a: np.ndarray, want_out: bool = True):
        a = _u32(a)
        n = a.shape[0]
        out = np.empty((n, self.cols), dtype=np.uint32) if want_out else None
        _load().oracle_stream_rows_u32(self._s, _ptr(a), _ptr(out) if out is not None else None, n,
                                       a.shape[1], self.cols)
        self.row += n
        return out

    def rows_f32(self, a: np.ndarray, want_out: bool = True, want_abs: bool = True):
        a = np.ascontiguousarray(a, dtype=np.float32)
        n = a.shape[0]
        out = np.empty((n, self.cols), dtype=np.float64) if want_out else None
        ab = np.empty((n, self.cols), dtype=np.float64) if want_abs else None
        _load().oracle_stream_rows_f32(self._s, _ptr(a), _ptr(out) if out is not None else None,
                                       _ptr(ab) if ab is not None else None, n, a.shape[1], self.cols)
        self.row += n
        return out, ab

    def colsums_u32(self) -> np.ndarray:
        out = np.empty(self.cols, dtype=np.uint32)
        _load().oracle_stream_colsums_u32(self._s, _ptr(out))
        return out

    def colsums_f64(self) -> np.ndarray:
        out = np.empty(self.cols, dtype=np.float64)
        _load().oracle_stream_colsums_f64(self._s, _ptr(out))
        return out


# ------------------------------------------------------------------------------------ region sums
def region_sum(a: np.ndarray, U: int, D: int, L: int, R: int):
    """S[U:D][L:R], by its double-sum definition; uint32 for integers, fp64 for floats."""
    if a.dtype == np.float32:
        a = np.ascontiguousarray(a)
        return _load().oracle_region_sum_f64(_ptr(a), a.shape[1], U, D, L, R)
    a = _u32(a)
    return _load().oracle_region_sum_u32(_ptr(a), a.shape[1], U, D, L, R)


def rect_sum(b: np.ndarray, u: int, d: int, l: int, r: int):
    """sum of a[i][j] for u < i <= d, l < j <= r, from four SAT entries; index -1 denotes the
    empty prefix (SAT value 0).  Evaluated in b's own arithmetic, left to right as P:48 writes it,
    ((b[d][r] - b[u][r]) - b[d][l]) + b[u][l] (reading R17): uint32 wraparound for integer b (an int),
    fp32 for float32 b (an np.float32), fp64 for float64 b."""
    if b.dtype in (np.uint32, np.int32):
        def at(i, j):
            return 0 if (i < 0 or j < 0) else int(b[i, j]) % (1 << 32)

        return (((at(d, r) - at(u, r)) - at(d, l)) + at(u, l)) % (1 << 32)
    z = b.dtype.type(0)

    def atf(i, j):
        return z if (i < 0 or j < 0) else b[i, j]

    return ((atf(d, r) - atf(u, r)) - atf(d, l)) + atf(u, l)


def box_sum(b: np.ndarray, rh: int, rw: int) -> np.ndarray:
    """Box filter from a SAT b: out[i][j] = the P:48 rectangle sum over rows
    (i-rh-1, min(i+rh, rows-1)] x cols (j-rw-1, min(j+rw, cols-1)], i.e. the input summed over the
    window [i-rh, i+rh] x [j-rw, j+rw] clipped to the matrix.  Evaluated in b's own arithmetic --
    uint32 wraparound for integer b, fp32 for float32 b -- left to right as written in P:48:
    ((b[d][r] - b[u][r]) - b[d][l]) + b[u][l] (reading R17); entries with index -1 are 0."""
    rows, cols = b.shape
    if b.dtype == np.float32:
        bp = np.zeros((rows + 1, cols + 1), dtype=np.float32)
    else:
        bp = np.zeros((rows + 1, cols + 1), dtype=np.uint32)
    bp[1:, 1:] = b if b.dtype == np.float32 else _u32(b)  # bp[x + 1][y + 1] = b[x][y]; index -1 -> 0
    i = np.arange(rows)
    j = np.arange(cols)
    u = np.maximum(i - rh - 1, -1) + 1
    d = np.minimum(i + rh, rows - 1) + 1
    l = np.maximum(j - rw - 1, -1) + 1
    r = np.minimum(j + rw, cols - 1) + 1
    with np.errstate(over="ignore"):
        out = bp[d][:, r] - bp[u][:, r]
        out = out - bp[d][:, l]
        out = out + bp[u][:, l]
    return out


# ------------------------------------------------------------------------------------ Table II
def table2(a: np.ndarray, TR: int, TC: int, I: int, J: int, with_gsat: bool = True) -> dict:
    """The per-tile sums of Table II for tile T(I,J) of TR x TC tiles (reading R5), each computed
    as the region sum S[..][..] that defines it.  Rows/cols beyond the matrix are absent (zero).
    ``with_gsat=False`` skips GSAT (TR*TC region sums) for large tiles."""
    rows, cols = a.shape
    r0, c0 = TR * I, TC * J
    r1, c1 = min(r0 + TR, rows) - 1, min(c0 + TC, cols) - 1
    S = lambda U, D, L, R: region_sum(a, U, D, L, R)  # noqa: E731
    out = {
        "LRS": [S(r0 + i, r0 + i, c0, c1) for i in range(r1 - r0 + 1)],
        "LCS": [S(r0, r1, c0 + j, c0 + j) for j in range(c1 - c0 + 1)],
        "LS": S(r0, r1, c0, c1),
        "GRS": [S(r0 + i, r0 + i, 0, c1) for i in range(r1 - r0 + 1)],
        "GCS": [S(0, r1, c0 + j, c0 + j) for j in range(c1 - c0 + 1)],
        "GS": S(0, r1, 0, c1),
        # GLS(I,J): the L-shaped region [0:r1] x [0:c1] minus [0:r0-1] x [0:c0-1] (Fig. 11 caption)
        "GLS": (S(r0, r1, 0, c1) + S(0, r0 - 1, c0, c1)) if a.dtype == np.float32
        else (S(r0, r1, 0, c1) + S(0, r0 - 1, c0, c1)) % (1 << 32),
        "GSAT": [[S(0, r0 + i, 0, c0 + j) for j in range(c1 - c0 + 1)] for i in range(r1 - r0 + 1)]
        if with_gsat else None,
    }
    return out


# ------------------------------------------------------------------------------------ Fig. 9 order
def tile_order(R: int, C: int) -> list[tuple[int, int]]:
    """Serial number -> tile (I, J) in diagonal-major order (Fig. 9): diagonals
    I+J = 0, 1, 2, ... in turn, I ascending within a diagonal, for an R x C tile grid (reading R6)."""
    order = []
    for d in range(R + C - 1):
        for I in range(max(0, d - C + 1), min(d, R - 1) + 1):
            order.append((I, d - I))
    return order


# ------------------------------------------------------------------------------------ strips
def strip_carry_u32(a_rows_above: np.ndarray, cols: int) -> np.ndarray:
    """Carry row of a strip: column sums (mod 2^32) of all rows above it (zero vector if none)."""
    s = Stream(cols)
    if a_rows_above.shape[0]:
        s.rows_u32(a_rows_above, want_out=False)
    c = s.colsums_u32()
    s.close()
    return c


# ------------------------------------------------------------------------------------ fp32 bound
F32_TOL_COEF = 1.2e-7


def f32_tolerance(absb: np.ndarray, rows: int, cols: int) -> np.ndarray:
    """BASELINE.json north_star: |gpu - oracle64| <= (rows+cols) * 1.2e-7 * absSAT (reading R10).
    rows/cols are the GLOBAL matrix sizes."""
    return (rows + cols) * F32_TOL_COEF * absb
