"""GPU parity at BASELINE.json's full sizes and shapes, plus the published per-tile aggregates.

* the 64K-column strip of configs[4] (rank 1 of 8 of a 64K x 64K matrix: 8192 x 65536 int32) with its
  carry row, through the strip-partition pipeline with the NCCL all-gather replaced by a local stack,
  every row against the streaming oracle fed with the rows above;
* the 64K x 64K single pass (configs[4] on one GPU), streamed row by row against the oracle;
* the 64K x 64K chained strip partition over 8 emulated ranks (configs[4] as bench.py projects it), every
  element;
* 32K x 32K fp32 with the cancellation distribution U[-1,1) (configs[3]);
* the aggregate words the kernels publish (Steps 2.A/2.B/3) against oracle.table2.
Needs a B200."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def sat():
    import paper_conf_ipps_emotofthni18_b200 as sat

    sat.set_tuning(-1, 0, 0)
    sat.set_max_ctas(0)
    yield sat
    sat.set_tuning(-1, 0, 0)
    sat.set_max_ctas(0)


MOD = 1 << 32


# ----------------------------------------------------------------------------- aggregates vs Table II
def _decode(words):
    return (words >> np.uint64(34)).astype(np.int64), ((words >> np.uint64(32)) & np.uint64(3)).astype(np.int64), \
        (words & np.uint64(0xFFFFFFFF)).astype(np.int64)


@pytest.mark.parametrize("variant,order,shape", [(0, 0, (150, 300)), (1, 0, (300, 300)), (1, 1, (257, 390)),
                                                 (3, 0, (150, 700)), (3, 0x200, (130, 1030))])
def test_published_aggregates_match_table2(sat, variant, order, shape):
    """Final state of every published word after one launch: row slots = prefix_i GRS(I,J), column slots =
    prefix_j GCS(I,J) (R5'), all inclusive; corner = GS(I,J) (inclusive) or GLS(I,J) (local, R8);
    one epoch throughout.  GRS / GCS / GS / GLS come from oracle.table2's region sums."""
    a = satgen.gen_host(*shape, seed=500 + variant, dist="u32")
    rows, cols = shape
    sat.set_tuning(variant, order, 0)
    try:
        x = torch.from_numpy(a).cuda()
        y = sat.sat(x)
        info, w = sat.debug_workspace()
    finally:
        sat.set_tuning(-1, 0, 0)
    assert (y.cpu().numpy() == oracle.sat_i32(a)).all()
    TR, TC, R, C = info["tile_rows"], info["tile_cols"], info["R"], info["C"]
    assert (R, C) == (-(-rows // TR), -(-cols // TC))
    n = R * C
    rs, cs, cn = w[: n * TR].reshape(n, TR), w[n * TR: n * (TR + TC)].reshape(n, TC), w[n * (TR + TC):]
    ep_r, kind_r, val_r = _decode(rs)
    ep_c, kind_c, val_c = _decode(cs)
    ep_n, kind_n, val_n = _decode(cn)
    epoch = int(ep_n[0])
    assert epoch >= 1 and (ep_r == epoch).all() and (ep_c == epoch).all() and (ep_n == epoch).all()
    assert (kind_r == 2).all() and (kind_c == 2).all(), "every row / column word ends inclusive"
    for I in range(R):
        for J in range(C):
            t = oracle.table2(a, TR, TC, I, J, with_gsat=False)
            k = I * C + J
            grs = np.cumsum(np.array(t["GRS"], dtype=np.int64)) % MOD
            gcs = np.cumsum(np.array(t["GCS"], dtype=np.int64)) % MOD
            nr, nc = len(grs), len(gcs)
            assert (val_r[k, :nr] == grs).all() and (val_r[k, nr:] == grs[-1]).all(), (I, J, "GRS")
            assert (val_c[k, :nc] == gcs).all() and (val_c[k, nc:] == gcs[-1]).all(), (I, J, "GCS")
            want = t["GS"] if kind_n[k] == 2 else t["GLS"]
            assert kind_n[k] in (1, 2) and val_n[k] == want % MOD, (I, J, "corner", kind_n[k])
    # edge tiles have nothing to look back at: their corner is GS at once (R10')
    for k in [0] + [J for J in range(C)] + [I * C for I in range(R)]:
        assert kind_n[k] == 2


# ----------------------------------------------------------------------------- full-size streaming checks
def _compare_rows(y, st, seed, dist, row0, rows_total, cols_total, chunk):
    n_rows = y.shape[0]
    worst = 0.0
    for r0 in range(0, n_rows, chunk):
        n = min(chunk, n_rows - r0)
        a = satgen.gen_host(n, y.shape[1], seed, dist, row0=row0 + r0)
        g = y[r0:r0 + n].cpu().numpy()
        if a.dtype == np.int32:
            want = st.rows_u32(a).view(np.int32)
            if not (g == want).all():
                bad = np.argwhere(g != want)[0]
                raise AssertionError(f"row {row0 + r0 + bad[0]} col {bad[1]}: {g[tuple(bad)]} != {want[tuple(bad)]}")
        else:
            want, absw = st.rows_f32(a)
            err = np.abs(g.astype(np.float64) - want)
            tol = oracle.f32_tolerance(absw, rows_total, cols_total)
            assert (err <= tol).all(), f"fp32 outside tolerance in rows {row0 + r0}..{row0 + r0 + n}"
            worst = max(worst, float((err / np.maximum(tol, 1e-300)).max()))
    return worst


@pytest.mark.slow
def test_64k_column_strip_with_carry(sat):
    """configs[4] strip shape: rank 1 of an 8-way split of 65536 x 65536 int32 (rows 8192..16383), its
    carry from rank 0's column sums (sat_strip_colsum -> stack -> sat_carry_prefix -> sat_compute with the
    carry, i.e. sat_compute_sharded with the all-gather done locally).  Every row vs the streaming oracle
    fed with rows 0..8191 first."""
    cols, h, seed = 65536, 8192, 4242
    top = torch.empty((h, cols), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(top, seed, "u32", row0=0)
    gathered = torch.stack([sat.strip_colsum(top), torch.zeros(cols, dtype=torch.int32, device="cuda")])
    del top
    carry = sat.carry_prefix(gathered, 1)
    strip = torch.empty((h, cols), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(strip, seed, "u32", row0=h)
    plan = sat.query_plan(sat.SAT_INT32, h, cols)
    assert (plan["tile_rows"], plan["tile_cols"]) == (64, 256)  # the production flat-tile kernel
    sat.sat(strip, out=strip, carry=carry)
    torch.cuda.synchronize()
    st = oracle.Stream(cols)
    for r0 in range(0, h, 1024):
        st.rows_u32(satgen.gen_host(1024, cols, seed, "u32", row0=r0), want_out=False)
    # the carry kernel's input equals the oracle's running column sums at row 8191
    assert (gathered[0].cpu().numpy().view(np.uint32) == st.colsums_u32()).all()
    _compare_rows(strip, st, seed, "u32", h, 2 * h, cols, 512)
    st.close()


@pytest.mark.slow
def test_64k_single_pass_every_element(sat):
    """The 64K x 64K int32 single pass on one GPU (in place, 16 GiB), every element vs the streaming oracle."""
    n, seed = 65536, 1447
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, seed, "u32")
    sat.sat(x, out=x)
    torch.cuda.synchronize()
    st = oracle.Stream(n)
    _compare_rows(x, st, seed, "u32", 0, n, n, 256)
    st.close()


@pytest.mark.slow
def test_full_32k_fp32_cancellation_every_element(sat):
    """32K x 32K fp32 with U[-1,1) inputs (sums cancel; the absSAT-scaled bound is the tight case)."""
    n, seed = 32768, 1449
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, seed, "fsym")
    y = sat.sat(x.view(torch.float32))
    torch.cuda.synchronize()
    del x
    st = oracle.Stream(n)
    worst = _compare_rows(y, st, seed, "fsym", 0, n, n, 1024)
    st.close()
    print(f"32K fp32 fsym: worst err/tol = {worst:.3e}")
    assert worst <= 1.0


@pytest.mark.slow
def test_64k_chained_8_ranks_every_element(sat):
    """configs[4] through the chained partition in the launch configuration bench.chain_projection times:
    65536 x 65536 int32 cut into 8 strips of 8192 rows, the 8 ranks emulated in one process (Chain.local,
    inbox pushes into the same HBM), each rank's kernel on the whole GPU in rank order, in place; then every
    element vs the streaming oracle."""
    n, N, seed = 65536, 8, 1447
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, seed, "u32")
    h = n // N
    chains = sat.Chain.local(N, n)
    try:
        for r in range(N):
            sat.sat_chained(x[r * h:(r + 1) * h], out=x[r * h:(r + 1) * h], chain=chains[r])
        torch.cuda.synchronize()
    finally:
        for c in chains:
            c.close()
    st = oracle.Stream(n)
    _compare_rows(x, st, seed, "u32", 0, n, n, 256)
    st.close()
