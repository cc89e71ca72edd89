"""Pins for the CPU oracle (oracle/): each check compares it with something other than itself --
the paper's worked example, the P:44 double-sum definition by brute force, closed forms, library
routines on the special cases that reduce to them, and invariants.  CPU only."""
import itertools
import math

import numpy as np
import pytest

import oracle
from conftest import read_golden_blocks

MOD = 1 << 32
RNG = np.random.default_rng(1447)


def brute_sat(a: np.ndarray) -> np.ndarray:
    """P:44 definition written as a double sum per entry (O(n^4)); exact Python ints."""
    rows, cols = a.shape
    ai = a.astype(np.int64) if a.dtype != np.float64 else a
    out = np.zeros((rows, cols), dtype=object)
    for i in range(rows):
        for j in range(cols):
            out[i, j] = int(ai[: i + 1, : j + 1].sum())
    return out


# ----------------------------------------------------------------------------- Figure 2
def test_fig2_column_prefix_and_sat_exact():
    g = read_golden_blocks("fig2_9x9.txt")
    a = np.array(g["input"], dtype=np.int32)
    c = oracle.col_prefix_u32(a)
    assert (c.astype(np.int64) == np.array(g["column_prefix"])).all()
    b = oracle.row_prefix_u32(c)
    assert (b.astype(np.int64) == np.array(g["sat"])).all()
    assert (oracle.sat_i32(a) == np.array(g["sat"])).all()
    assert int(oracle.sat_u32(a)[8, 8]) == 71  # the total printed in Fig. 2


def test_fig2_fp64_path_exact():
    g = read_golden_blocks("fig2_9x9.txt")
    a = np.array(g["input"], dtype=np.float32)
    b, ab = oracle.sat_f32(a)
    assert (b == np.array(g["sat"], dtype=np.float64)).all()
    assert (ab == b).all()  # nonnegative input: |a| = a


# ----------------------------------------------------------------------------- brute force
def _random_shapes(n):
    shapes = [(1, 1), (1, 16), (16, 1), (1, 7), (9, 1), (16, 16), (2, 3), (3, 2)]
    while len(shapes) < n:
        shapes.append((int(RNG.integers(1, 17)), int(RNG.integers(1, 17))))
    return shapes


@pytest.mark.parametrize("chunk", range(4))
def test_brute_force_uint32_full_range(chunk):
    for rows, cols in _random_shapes(220)[chunk::4]:
        a = RNG.integers(0, MOD, size=(rows, cols), dtype=np.uint64).astype(np.uint32)
        ref = brute_sat(a)
        got = oracle.sat_u32(a)
        for i in range(rows):
            for j in range(cols):
                assert int(got[i, j]) == ref[i, j] % MOD, (rows, cols, i, j)


def test_brute_force_int32_signed_small():
    for rows, cols in _random_shapes(60):
        a = RNG.integers(-1000, 1000, size=(rows, cols)).astype(np.int32)
        ref = brute_sat(a).astype(np.int64)
        assert (oracle.sat_i32(a).astype(np.int64) == ref).all()


def test_brute_force_fp64_within_sequential_bound():
    """fp64 oracle vs exactly rounded rectangle sums (math.fsum): the error of a sum of depth d is
    <= d * 2^-53 * sum|a| (first order); depth here <= rows + cols."""
    for rows, cols in _random_shapes(60):
        a = (RNG.random((rows, cols), dtype=np.float32) * 2 - 1).astype(np.float32)
        b, ab = oracle.sat_f32(a)
        for i in range(rows):
            for j in range(cols):
                blk = a[: i + 1, : j + 1].astype(np.float64).ravel()
                exact = math.fsum(blk)
                absexact = math.fsum(np.abs(blk))
                assert abs(b[i, j] - exact) <= (i + j + 2) * 2.0 ** -52 * absexact + 1e-300
                assert abs(ab[i, j] - absexact) <= (i + j + 2) * 2.0 ** -52 * absexact + 1e-300


def test_fp64_exact_for_integers():
    for rows, cols in _random_shapes(40):
        a = RNG.integers(-(2 ** 20), 2 ** 20, size=(rows, cols)).astype(np.float32)
        b, _ = oracle.sat_f32(a)
        assert (b == brute_sat(a.astype(np.float64)).astype(np.float64)).all()
    a = RNG.integers(-(2 ** 30), 2 ** 30, size=(12, 13)).astype(np.float64)
    assert (oracle.sat_f64(a) == brute_sat(a).astype(np.float64)).all()


# ----------------------------------------------------------------------------- rectangle formula
def test_rectangle_formula_all_rectangles():
    a = RNG.integers(0, MOD, size=(7, 8), dtype=np.uint64).astype(np.uint32)
    b = oracle.sat_u32(a)
    rows, cols = a.shape
    for u, d in itertools.combinations(range(-1, rows), 2):
        for l, r in itertools.combinations(range(-1, cols), 2):
            want = int(a[u + 1: d + 1, l + 1: r + 1].astype(np.int64).sum()) % MOD
            assert oracle.rect_sum(b, u, d, l, r) == want
            assert oracle.region_sum(a, u + 1, d, l + 1, r) == want



def brute_box(a: np.ndarray, rh: int, rw: int) -> np.ndarray:
    """Window sums by direct summation of the clipped window (exact Python ints)."""
    rows, cols = a.shape
    ai = a.astype(np.int64)
    out = np.zeros((rows, cols), dtype=object)
    for i in range(rows):
        for j in range(cols):
            out[i, j] = int(ai[max(0, i - rh): i + rh + 1, max(0, j - rw): j + rw + 1].sum())
    return out


@pytest.mark.parametrize("shape,rh,rw", [((1, 1), 0, 0), ((7, 9), 1, 2), ((12, 5), 3, 0), ((6, 6), 10, 10),
                                         ((9, 13), 0, 4), ((16, 11), 2, 7)])
def test_box_sum_is_the_clipped_window_sum(shape, rh, rw):
    a = RNG.integers(0, MOD, size=shape, dtype=np.uint64).astype(np.uint32)
    got = oracle.box_sum(oracle.sat_u32(a), rh, rw)
    want = np.vectorize(lambda x: x % MOD)(brute_box(a, rh, rw)).astype(np.uint64)
    assert (got.astype(np.uint64) == want).all()


def test_box_sum_fp32_exact_regime_and_association():
    # small integers in fp32: every SAT entry and every partial of the P:48 formula is exact
    a = RNG.integers(0, 4, size=(23, 31)).astype(np.float32)
    b = oracle.sat_f64(a).astype(np.float32)
    got = oracle.box_sum(b, 2, 3)
    assert got.dtype == np.float32
    assert (got.astype(np.float64) == brute_box(a, 2, 3).astype(np.float64)).all()
    # evaluation order is ((drr - urr) - dll) + ull in fp32: check one entry against that by hand
    b = RNG.standard_normal((5, 6)).astype(np.float32) * np.float32(1e4)
    o = oracle.box_sum(b, 1, 1)
    i, j = 3, 4  # u = 1, d = 4, l = 2, r = 5
    want = ((b[4, 5] - b[1, 5]) - b[4, 2]) + b[1, 2]
    assert o[i, j] == want

# ----------------------------------------------------------------------------- closed forms
def test_all_ones():
    a = np.ones((37, 53), dtype=np.int32)
    i, j = np.indices(a.shape)
    assert (oracle.sat_i32(a) == (i + 1) * (j + 1)).all()


def test_impulse():
    for p, q in [(0, 0), (5, 9), (36, 52), (20, 0)]:
        a = np.zeros((37, 53), dtype=np.int32)
        a[p, q] = 7
        i, j = np.indices(a.shape)
        assert (oracle.sat_i32(a) == 7 * ((i >= p) & (j >= q))).all()


def test_rank_one_mod_2_32():
    u = RNG.integers(0, MOD, size=29, dtype=np.uint64)
    v = RNG.integers(0, MOD, size=31, dtype=np.uint64)
    a = ((u[:, None] * v[None, :]) % MOD).astype(np.uint32)
    U = np.cumsum(u.astype(object)) % MOD
    V = np.cumsum(v.astype(object)) % MOD
    want = (U[:, None] * V[None, :]) % MOD
    assert (oracle.sat_u32(a).astype(object) == want).all()


def test_single_row_and_column_are_1d_prefix_sums():
    x = RNG.integers(-(2 ** 31), 2 ** 31, size=1000).astype(np.int32)
    want = np.cumsum(x.astype(np.int64)) % MOD
    assert (oracle.sat_u32(x[None, :])[0].astype(np.int64) == want).all()
    assert (oracle.sat_u32(x[:, None])[:, 0].astype(np.int64) == want).all()
    f = RNG.random(500).astype(np.float32)
    b, _ = oracle.sat_f32(f[None, :])
    assert np.allclose(b[0], np.cumsum(f.astype(np.float64)), rtol=0, atol=1e-9)


def test_transpose_and_linearity():
    a = RNG.integers(0, MOD, size=(23, 41), dtype=np.uint64).astype(np.uint32)
    c = RNG.integers(0, MOD, size=(23, 41), dtype=np.uint64).astype(np.uint32)
    assert (oracle.sat_u32(np.ascontiguousarray(a.T)) == oracle.sat_u32(a).T).all()
    with np.errstate(over="ignore"):
        lhs = oracle.sat_u32(a + c * np.uint32(3))
        rhs = oracle.sat_u32(a) + oracle.sat_u32(c) * np.uint32(3)
    assert (lhs == rhs).all()


# ----------------------------------------------------------------------------- invariants
def test_total_and_inverse_identity():
    a = RNG.integers(0, MOD, size=(64, 80), dtype=np.uint64).astype(np.uint32)
    b = oracle.sat_u32(a).astype(np.int64)
    assert b[-1, -1] % MOD == int(a.astype(np.int64).sum()) % MOD
    bp = np.zeros((65, 81), dtype=np.int64)
    bp[1:, 1:] = b
    back = (bp[1:, 1:] - bp[:-1, 1:] - bp[1:, :-1] + bp[:-1, :-1]) % MOD
    assert (back == a.astype(np.int64)).all()


# ----------------------------------------------------------------------------- streaming form
def test_stream_matches_definition_and_carry():
    rows, cols = 45, 33
    a = RNG.integers(0, MOD, size=(rows, cols), dtype=np.uint64).astype(np.uint32)
    ref = brute_sat(a)
    s = oracle.Stream(cols)
    got = np.concatenate([s.rows_u32(a[r0:r0 + 7]) for r0 in range(0, rows, 7)])
    assert s.row == rows
    assert all(int(got[i, j]) == ref[i, j] % MOD for i in range(rows) for j in range(cols))
    assert (s.colsums_u32().astype(np.int64) == a.astype(np.int64).sum(axis=0) % MOD).all()
    s.close()
    # strip carry = column sums of the rows above the strip
    carry = oracle.strip_carry_u32(a[:20], cols)
    assert (carry.astype(np.int64) == a[:20].astype(np.int64).sum(axis=0) % MOD).all()
    assert (oracle.strip_carry_u32(a[:0], cols) == 0).all()


def test_stream_f32_matches_in_memory():
    a = (RNG.random((40, 29), dtype=np.float32) * 2 - 1).astype(np.float32)
    b, ab = oracle.sat_f32(a)
    s = oracle.Stream(29)
    parts = [s.rows_f32(a[r0:r0 + 9]) for r0 in range(0, 40, 9)]
    sb = np.concatenate([p[0] for p in parts])
    sab = np.concatenate([p[1] for p in parts])
    # same two passes in the same order: identical bits
    assert (sb == b).all() and (sab == ab).all()
    assert np.allclose(s.colsums_f64(), a.astype(np.float64).sum(axis=0), rtol=0, atol=1e-12)


# ----------------------------------------------------------------------------- Table II (R5), P:150/P:162/P:233/P:241
@pytest.mark.parametrize("shape,TR,TC", [((13, 17), 4, 5), ((12, 12), 4, 4), ((9, 9), 3, 3)])
def test_table2_relations(shape, TR, TC):
    a = RNG.integers(0, MOD, size=shape, dtype=np.uint64).astype(np.uint32)
    b = oracle.sat_u32(a).astype(np.int64)
    rows, cols = shape
    R, C = -(-rows // TR), -(-cols // TC)
    T = {(I, J): oracle.table2(a, TR, TC, I, J) for I in range(R) for J in range(C)}
    for (I, J), t in T.items():
        r0, c0 = TR * I, TC * J
        r1, c1 = min(r0 + TR, rows) - 1, min(c0 + TC, cols) - 1
        # GS(I,J) is the bottom-right corner of GSAT(I,J); GSAT entries are SAT entries
        assert t["GS"] == b[r1, c1] % MOD
        assert all(t["GSAT"][i][j] == b[r0 + i, c0 + j] % MOD
                   for i in range(r1 - r0 + 1) for j in range(c1 - c0 + 1))
        # GRS/GCS = adjacent differences of GSAT's rightmost column / bottom row
        for i in range(r1 - r0 + 1):
            above = b[r0 + i - 1, c1] if r0 + i > 0 else 0
            assert t["GRS"][i] == (b[r0 + i, c1] - above) % MOD
        for j in range(c1 - c0 + 1):
            left = b[r1, c0 + j - 1] if c0 + j > 0 else 0
            assert t["GCS"][j] == (b[r1, c0 + j] - left) % MOD
        # GRS(I,J) = GRS(I,J-1) + LRS(I,J); column analogue
        lrs, lcs = t["LRS"], t["LCS"]
        grs_l = T[(I, J - 1)]["GRS"] if J > 0 else [0] * len(lrs)
        gcs_u = T[(I - 1, J)]["GCS"] if I > 0 else [0] * len(lcs)
        assert all(t["GRS"][i] == (grs_l[i] + lrs[i]) % MOD for i in range(len(lrs)))
        assert all(t["GCS"][j] == (gcs_u[j] + lcs[j]) % MOD for j in range(len(lcs)))
        # Fig. 11 / P:241 (Step 3.1): GLS(I,J) = sum of GRS(I,J-1) + LRS(I,J) + GCS(I-1,J)
        assert t["GLS"] == (sum(grs_l) + sum(lrs) + sum(gcs_u)) % MOD
        # Step 3.3: GS(I,J) = GS(I-1,J-1) + GLS(I,J)
        gs_d = T[(I - 1, J - 1)]["GS"] if (I > 0 and J > 0) else 0
        assert t["GS"] == (gs_d + t["GLS"]) % MOD
        assert t["LS"] == sum(lrs) % MOD == sum(lcs) % MOD
        # P:150 injection rule: SAT of the tile with GRS(I,J-1) added to its left column,
        # GCS(I-1,J) to its top row and GS(I-1,J-1) to its corner equals GSAT(I,J)
        u = a[r0:r1 + 1, c0:c1 + 1].astype(np.int64).copy()
        u[:, 0] += np.array(grs_l, dtype=np.int64)
        u[0, :] += np.array(gcs_u, dtype=np.int64)
        u[0, 0] += gs_d
        assert (oracle.sat_u32((u % MOD).astype(np.uint32)).astype(np.int64)
                == b[r0:r1 + 1, c0:c1 + 1] % MOD).all()


# ----------------------------------------------------------------------------- Figure 9
def test_fig9_tile_order():
    table = read_golden_blocks("fig9_order_5x5.txt")[None]
    order = oracle.tile_order(5, 5)
    for s, (I, J) in enumerate(order):
        assert table[I][J] == s
    # the P:186 closed form disagrees with the figure exactly where I+J >= n/W (reading R6)
    bad = [(I, J) for I in range(5) for J in range(5) if (I + J) * (I + J + 1) // 2 + I != table[I][J]]
    assert len(bad) == 10 and all(I + J >= 5 for I, J in bad)


@pytest.mark.parametrize("R,C", [(1, 1), (1, 7), (6, 1), (4, 9), (9, 4), (16, 16)])
def test_tile_order_is_topological(R, C):
    order = oracle.tile_order(R, C)
    assert sorted(order) == [(I, J) for I in range(R) for J in range(C)]
    pos = {t: s for s, t in enumerate(order)}
    for (I, J), s in pos.items():
        for dep in [(I, J - 1), (I - 1, J), (I - 1, J - 1)]:
            if dep in pos:
                assert pos[dep] < s


# ----------------------------------------------------------------------------- fp32 tolerance (R10)
def test_f32_tolerance_accepts_fp32_sat_and_rejects_perturbation():
    a = (RNG.random((300, 200), dtype=np.float32) * 2 - 1).astype(np.float32)
    b, ab = oracle.sat_f32(a)
    # an fp32 column-then-row computation (a different precision) must pass the bound ...
    f32 = np.cumsum(np.cumsum(a, axis=0, dtype=np.float32), axis=1, dtype=np.float32)
    tol = oracle.f32_tolerance(ab, *a.shape)
    assert (np.abs(f32.astype(np.float64) - b) <= tol).all()
    # ... and the bound is not vacuous: a one-ulp-of-the-total error at a late entry fails it
    bad = f32.astype(np.float64).copy()
    bad[150, 100] += 4 * tol[150, 100] + 1e-3
    assert not (np.abs(bad - b) <= tol).all()


# ----------------------------------------------------------------------------- fp32 / fp64 branches
def test_region_sum_f64_against_fsum():
    """oracle_region_sum_f64 (S[U:D][L:R] of P:128 for float input) vs the exactly rounded sum."""
    a = (RNG.random((11, 14), dtype=np.float32) * 2 - 1).astype(np.float32)
    rows, cols = a.shape
    for U, D in itertools.combinations_with_replacement(range(rows), 2):
        for L, R in [(0, cols - 1), (3, 3), (2, 9), (13, 13), (5, 12)]:
            blk = a[U:D + 1, L:R + 1].astype(np.float64).ravel()
            got = oracle.region_sum(a, U, D, L, R)
            assert abs(got - math.fsum(blk)) <= blk.size * 2.0 ** -53 * math.fsum(np.abs(blk)) + 1e-300
    assert oracle.region_sum(a, 5, 4, 0, 3) == 0.0  # empty range (D < U): the zero aggregates of R5
    assert oracle.region_sum(a, 0, 3, 7, 6) == 0.0
    # integers below 2^24 (exact in fp32 and in every fp64 partial): equals the integer region sum
    ai = RNG.integers(-(2 ** 20), 2 ** 20, size=(9, 10)).astype(np.float32)
    assert oracle.region_sum(ai, 2, 7, 1, 8) == float(ai[2:8, 1:9].astype(np.int64).sum())


def test_rect_sum_float_branches():
    """rect_sum on float32 / float64 SATs: the P:48 formula in the SAT's own precision (R17)."""
    a = RNG.integers(0, 4, size=(9, 12)).astype(np.float64)
    b64 = oracle.sat_f64(a)  # exact: small integers
    b32 = b64.astype(np.float32)
    rows, cols = a.shape
    for u, d in itertools.combinations(range(-1, rows), 2):
        for l, r in itertools.combinations(range(-1, cols), 2):
            want = float(a[u + 1: d + 1, l + 1: r + 1].sum())
            g32 = oracle.rect_sum(b32, u, d, l, r)
            assert isinstance(g32, np.float32) and float(g32) == want
            assert oracle.rect_sum(b64, u, d, l, r) == want
    # association: ((drr - urr) - dll) + ull, each step rounded to fp32
    bf = (RNG.standard_normal((6, 7)) * 1e4).astype(np.float32)
    want = ((bf[5, 6] - bf[2, 6]) - bf[5, 3]) + bf[2, 3]
    assert oracle.rect_sum(bf, 2, 5, 3, 6) == want
    assert oracle.rect_sum(bf, -1, 5, -1, 6) == bf[5, 6]


def test_table2_float_branch_against_fsum():
    """Table II of an fp32 matrix (fp64 region sums): every entry within the fp64 summation bound of
    the exactly rounded region sum, and the P:162 / P:233 / P:241 relations to fp64 rounding."""
    a = (RNG.random((10, 13), dtype=np.float32) * 2 - 1).astype(np.float32)
    TR, TC = 4, 5
    rows, cols = a.shape
    eps = 64 * 2.0 ** -53 * float(np.abs(a.astype(np.float64)).sum())
    fs = lambda U, D, L, R: math.fsum(a[U:D + 1, L:R + 1].astype(np.float64).ravel()) if (D >= U and R >= L) else 0.0  # noqa: E731
    T = {(I, J): oracle.table2(a, TR, TC, I, J) for I in range(3) for J in range(3)}
    for (I, J), t in T.items():
        r0, c0 = TR * I, TC * J
        r1, c1 = min(r0 + TR, rows) - 1, min(c0 + TC, cols) - 1
        assert abs(t["GS"] - fs(0, r1, 0, c1)) <= eps
        assert abs(t["LS"] - fs(r0, r1, c0, c1)) <= eps
        assert abs(t["GLS"] - (fs(0, r1, 0, c1) - fs(0, r0 - 1, 0, c0 - 1))) <= eps  # the L-shaped region
        for i in range(r1 - r0 + 1):
            assert abs(t["GRS"][i] - fs(r0 + i, r0 + i, 0, c1)) <= eps
            assert abs(t["LRS"][i] - fs(r0 + i, r0 + i, c0, c1)) <= eps
        for j in range(c1 - c0 + 1):
            assert abs(t["GCS"][j] - fs(0, r1, c0 + j, c0 + j)) <= eps
        gs_d = T[(I - 1, J - 1)]["GS"] if (I > 0 and J > 0) else 0.0
        assert abs(t["GS"] - (gs_d + t["GLS"])) <= eps  # Step 3.3
        grs_l = T[(I, J - 1)]["GRS"] if J > 0 else [0.0] * len(t["LRS"])
        assert all(abs(t["GRS"][i] - (grs_l[i] + t["LRS"][i])) <= eps for i in range(len(t["LRS"])))


def test_moments_f32_against_fsum_and_closed_form():
    """Variance-shadow-map moments (ref. [8]): SAT(a) and SAT(a*a) vs exactly rounded sums; a
    constant c gives (i+1)(j+1)c and (i+1)(j+1)c^2."""
    a = (RNG.random((13, 17), dtype=np.float32) * 2 - 1).astype(np.float32)
    s1, ab1, s2, ab2 = oracle.moments_f32(a)
    a64 = a.astype(np.float64)
    for i in range(a.shape[0]):
        for j in range(a.shape[1]):
            blk = a64[: i + 1, : j + 1].ravel()
            sq = blk * blk
            assert abs(s1[i, j] - math.fsum(blk)) <= (i + j + 2) * 2.0 ** -52 * math.fsum(np.abs(blk))
            assert abs(ab1[i, j] - math.fsum(np.abs(blk))) <= (i + j + 2) * 2.0 ** -52 * math.fsum(np.abs(blk))
            assert abs(s2[i, j] - math.fsum(sq)) <= (i + j + 2) * 2.0 ** -52 * math.fsum(sq)
    assert (ab2 == s2).all()
    c = np.full((6, 9), 0.75, dtype=np.float32)
    i, j = np.indices(c.shape)
    s1, _, s2, _ = oracle.moments_f32(c)
    assert (s1 == (i + 1) * (j + 1) * 0.75).all() and (s2 == (i + 1) * (j + 1) * 0.5625).all()
