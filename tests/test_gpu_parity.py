"""GPU parity: libsat's CUDA path (through the C ABI) vs the CPU oracle, element by element on the
same seeded inputs.  int32: bit-exact (uint32 wraparound).  fp32: |gpu - oracle64| <=
(rows+cols) * 1.2e-7 * absSAT (BASELINE.json north_star; R10); bit-exact in the exact
regime (inputs in {0..3}, every partial sum an integer < 2^24).  Needs a B200."""
import numpy as np
import pytest

import oracle
import satgen
from conftest import read_golden_blocks

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


def dev_copy(a: np.ndarray, pitch: int | None = None, offset_words: int = 0):
    """Upload a host matrix into a fresh device buffer with row stride `pitch` (pad = sentinel)."""
    rows, cols = a.shape
    pitch = cols if pitch is None else pitch
    t = torch.empty(rows * pitch + offset_words + 64, dtype=torch.int32, device="cuda")
    t.fill_(0x5A5A5A5A)
    flat = t[offset_words: offset_words + rows * pitch]
    m = flat.view(rows, pitch)[:, :cols]
    m.copy_(torch.from_numpy(a.view(np.int32)).to("cuda"))
    if a.dtype == np.float32:
        return t, m.view(torch.float32)
    return t, m


def run_sat(sat, a: np.ndarray, pitch=None, inplace=False, carry=None, offset_words=0):
    buf, src = dev_copy(a, pitch, offset_words)
    if inplace:
        out = src
    else:
        obuf, out = dev_copy(np.zeros_like(a), pitch, offset_words)
    sat.sat(src, out=out, carry=carry)
    torch.cuda.synchronize()
    res = out.cpu().numpy()
    if pitch is not None and pitch > a.shape[1]:
        # pad words of every row are never written
        ob = (buf if inplace else obuf)
        full = ob[offset_words: offset_words + a.shape[0] * pitch].view(a.shape[0], pitch)
        assert (full[:, a.shape[1]:] == 0x5A5A5A5A).all(), "pad elements were written"
    return res


def assert_i32_exact(got, a):
    want = oracle.sat_i32(a)
    if not (got.view(np.int32) == want).all():
        bad = np.argwhere(got.view(np.int32) != want)
        raise AssertionError(f"{len(bad)} mismatches of {a.size}; first at {bad[0].tolist()}: "
                             f"got {got.view(np.int32)[tuple(bad[0])]} want {want[tuple(bad[0])]}")


def assert_f32_tol(got, a, rows=None, cols=None):
    b, ab = oracle.sat_f32(a)
    rows = a.shape[0] if rows is None else rows
    cols = a.shape[1] if cols is None else cols
    tol = oracle.f32_tolerance(ab, rows, cols)
    err = np.abs(got.astype(np.float64) - b)
    if not (err <= tol).all():
        i = np.unravel_index(np.argmax(err - tol), err.shape)
        raise AssertionError(f"fp32 outside tolerance at {i}: err {err[i]} tol {tol[i]}")


SHAPES = [(1, 1), (1, 5000), (5000, 1), (9, 9), (64, 128), (65, 129), (129, 257), (256, 256),
          (300, 4096), (1009, 2003), (2048, 33), (33, 2048), (777, 1500)]


# ----------------------------------------------------------------------------------- generator
@pytest.mark.parametrize("dist", ["u32", "u8", "u2", "f01", "fsym", "fu2"])
def test_device_generator_matches_host(dist):
    rows, cols, pitch = 123, 517, 520
    t = torch.zeros(rows, pitch, dtype=torch.int32, device="cuda")
    satgen.fill_device(t.data_ptr(), rows, cols, pitch, 1447, dist, row0=77,
                       stream=torch.cuda.current_stream().cuda_stream)
    host = satgen.gen_host(rows, cols, 1447, dist, row0=77)
    assert (t.cpu().numpy()[:, :cols] == host.view(np.int32)).all()
    assert (t.cpu().numpy()[:, cols:] == 0).all()


# ----------------------------------------------------------------------------------- int32
def test_fig2_worked_example(sat):
    g = read_golden_blocks("fig2_9x9.txt")
    a = np.array(g["input"], dtype=np.int32)
    got = run_sat(sat, a)
    assert (got == np.array(g["sat"])).all()


@pytest.mark.parametrize("shape", SHAPES)
def test_int32_bit_exact(sat, shape):
    a = satgen.gen_host(*shape, seed=1447 + shape[0], dist="u32")
    assert_i32_exact(run_sat(sat, a), a)


@pytest.mark.parametrize("variant", range(20))
@pytest.mark.parametrize("order", [0, 1, 0x400])
def test_int32_every_variant_and_order(sat, variant, order):
    if variant >= sat.num_variants():
        pytest.skip("no such variant")
    sat.set_tuning(variant, order, 0)
    try:
        sat.sat(torch.zeros((8, 8), dtype=torch.int32, device="cuda"))
    except sat.SatError as e:
        sat.set_tuning(-1, 0, 0)
        if e.status == 3:  # SAT_ERR_UNSUPPORTED: a variant for another input type (u8 integral images)
            pytest.skip(str(e))
        raise
    try:
        for shape in [(1000, 1000), (257, 3000), (4096, 130), (100, 2050)]:
            a = satgen.gen_host(*shape, seed=99 + variant, dist="u32")
            assert_i32_exact(run_sat(sat, a), a)
    finally:
        sat.set_tuning(-1, 0, 0)


# production flat-tile kernel (variant 3, 64 x 256 tiles, 2-tile-group order) and the 128 x 128 kernel
# (variant 1), forced at sizes where auto-selection would pick another kernel: every data path of the
# ABI contract
FLAT = [(3, 0x200), (3, 0), (1, 0x200), (1, 0)]


@pytest.mark.parametrize("variant,order", FLAT)
def test_flat_tile_kernel_contract(sat, variant, order):
    sat.set_tuning(variant, order, 0)
    try:
        a = satgen.gen_host(700, 1300, seed=71, dist="u32")
        assert_i32_exact(run_sat(sat, a), a)                        # TMA path, ragged last tile column
        assert_i32_exact(run_sat(sat, a, pitch=1304), a)            # pitch pad untouched (TMA)
        assert_i32_exact(run_sat(sat, a, pitch=1301), a)            # generic loads/stores (pitch*4 % 16 != 0)
        assert_i32_exact(run_sat(sat, a, offset_words=1), a)        # misaligned base: generic path
        assert_i32_exact(run_sat(sat, a, inplace=True), a)          # src == dst
        assert_i32_exact(run_sat(sat, a, pitch=1304, inplace=True), a)
        b = satgen.gen_host(65, 3001, seed=72, dist="u32")         # 2 tile rows, 12 tile columns, ragged both ways
        assert_i32_exact(run_sat(sat, b, pitch=3004), b)
        f = satgen.gen_host(1000, 1537, seed=73, dist="fsym")
        assert_f32_tol(run_sat(sat, f), f)
        e = satgen.gen_host(640, 2048, seed=74, dist="fu2")         # exact regime: fp32 bit-exact
        assert (run_sat(sat, e).astype(np.float64) == oracle.sat_f32(e)[0]).all()
        # carry row (the strip-partitioned path): lower strip of a stacked SAT
        rows, cols, top = 900, 1100, 357
        c = satgen.gen_host(rows, cols, seed=75, dist="u32")
        full = oracle.sat_i32(c)
        carry = torch.from_numpy(np.ascontiguousarray(full[top - 1])).cuda()
        assert (run_sat(sat, np.ascontiguousarray(c[top:]), carry=carry) == full[top:]).all()
        # forward progress with few persistent CTAs
        for n in [1, 3]:
            sat.set_max_ctas(n)
            try:
                assert_i32_exact(run_sat(sat, a), a)
            finally:
                sat.set_max_ctas(0)
    finally:
        sat.set_tuning(-1, 0, 0)


def test_int32_pitch_pad_untouched(sat):
    a = satgen.gen_host(500, 1000, seed=5, dist="u32")
    assert_i32_exact(run_sat(sat, a, pitch=1024), a)   # TMA path (pitch*4 % 16 == 0)
    assert_i32_exact(run_sat(sat, a, pitch=1003), a)   # generic path (pitch*4 % 16 != 0)


def test_int32_misaligned_base_uses_generic_path(sat):
    a = satgen.gen_host(300, 700, seed=6, dist="u32")
    assert_i32_exact(run_sat(sat, a, offset_words=1), a)


@pytest.mark.parametrize("cols", [997, 998, 999, 1000, 1001])
@pytest.mark.parametrize("inplace", [False, True])
def test_ragged_width_with_pad(sat, cols, inplace):
    """Row widths that are not a multiple of 4 elements: pad words of a 16-byte-aligned pitch must stay
    untouched by the TMA path."""
    a = satgen.gen_host(333, cols, seed=cols, dist="u32")
    assert_i32_exact(run_sat(sat, a, pitch=1008, inplace=inplace), a)


def test_int32_in_place(sat):
    a = satgen.gen_host(1111, 999, seed=8, dist="u32")
    assert_i32_exact(run_sat(sat, a, inplace=True), a)
    assert_i32_exact(run_sat(sat, a, pitch=1000, inplace=True), a)


def test_int32_small_values_and_u8(sat):
    for dist in ["u8", "u2"]:
        a = satgen.gen_host(1500, 1700, seed=11, dist=dist)
        assert_i32_exact(run_sat(sat, a), a)


def test_int32_deterministic_repeats(sat):
    a = satgen.gen_host(2048, 2048, seed=12, dist="u32")
    _, src = dev_copy(a)
    first = sat.sat(src)
    for _ in range(50):
        again = sat.sat(src)
        assert torch.equal(first, again)
    assert_i32_exact(first.cpu().numpy(), a)


def test_single_cta_forward_progress(sat):
    """One persistent CTA must still complete every tile (correct for any CTA assignment)."""
    sat.set_max_ctas(1)
    try:
        for order in [0, 1]:
            sat.set_tuning(-1, order, 0)
            a = satgen.gen_host(700, 900, seed=13, dist="u32")
            assert_i32_exact(run_sat(sat, a), a)
    finally:
        sat.set_max_ctas(0)
        sat.set_tuning(-1, 0, 0)


def test_few_ctas(sat):
    for n in [2, 3, 7]:
        sat.set_max_ctas(n)
        try:
            a = satgen.gen_host(1000, 1300, seed=20 + n, dist="u32")
            assert_i32_exact(run_sat(sat, a), a)
        finally:
            sat.set_max_ctas(0)


def test_concurrent_streams(sat):
    shapes = [(1500, 1500), (999, 2500), (3000, 700)]
    arrs = [satgen.gen_host(*s, seed=30 + i, dist="u32") for i, s in enumerate(shapes)]
    streams = [torch.cuda.Stream() for _ in shapes]
    srcs = [torch.from_numpy(a).cuda() for a in arrs]
    torch.cuda.synchronize()
    outs = []
    for rep in range(3):
        outs = []
        for s, x in zip(streams, srcs):
            with torch.cuda.stream(s):
                outs.append(sat.sat(x))
        torch.cuda.synchronize()
    for o, a in zip(outs, arrs):
        assert_i32_exact(o.cpu().numpy(), a)


def test_empty_and_degenerate(sat):
    x = torch.empty((0, 10), dtype=torch.int32, device="cuda")
    assert sat.sat(x).shape == (0, 10)
    x = torch.empty((10, 0), dtype=torch.int32, device="cuda")
    assert sat.sat(x).shape == (10, 0)
    z = np.zeros((513, 257), dtype=np.int32)
    assert (run_sat(sat, z) == 0).all()
    ones = np.ones((300, 400), dtype=np.int32)
    i, j = np.indices(ones.shape)
    assert (run_sat(sat, ones) == (i + 1) * (j + 1)).all()


def test_error_codes_on_gpu(sat):
    from paper_conf_ipps_emotofthni18_b200 import _lib

    L = _lib.lib()
    t = torch.zeros(4096, dtype=torch.int32, device="cuda")
    base = t.data_ptr()
    assert L.sat_compute(0, base + 2, base + 8192, 4, 8, 8, None, None) == 2  # MISALIGNED
    assert L.sat_compute(0, base, base + 16, 4, 8, 8, None, None) == 1       # partial overlap
    with pytest.raises(TypeError):
        sat.sat(torch.zeros((4, 4), dtype=torch.int64, device="cuda"))


# ----------------------------------------------------------------------------------- fp32
@pytest.mark.parametrize("shape", [(1, 4000), (4000, 1), (9, 9), (256, 256), (1009, 2003), (777, 1500)])
@pytest.mark.parametrize("dist", ["f01", "fsym"])
def test_fp32_tolerance(sat, shape, dist):
    a = satgen.gen_host(*shape, seed=2024 + shape[1], dist=dist)
    assert_f32_tol(run_sat(sat, a), a)


def test_fp32_exact_regime_bit_exact(sat):
    a = satgen.gen_host(2048, 2048, seed=77, dist="fu2")
    got = run_sat(sat, a)
    want = oracle.sat_u32(a.astype(np.int32)).astype(np.float64)
    assert want.max() < 2 ** 24
    assert (got.astype(np.float64) == want).all()


def test_fp32_in_place_and_pitch(sat):
    a = satgen.gen_host(600, 900, seed=78, dist="fsym")
    assert_f32_tol(run_sat(sat, a, inplace=True, pitch=904), a)
    assert_f32_tol(run_sat(sat, a, pitch=901), a)


# ----------------------------------------------------------------------------------- carry row
@pytest.mark.parametrize("dist", ["u32", "fsym"])
def test_carry_row_equals_lower_strip_of_stacked_sat(sat, dist):
    rows, cols, top = 900, 1100, 357
    a = satgen.gen_host(rows, cols, seed=41, dist=dist)
    if dist == "u32":
        full = oracle.sat_i32(a)
        carry = torch.from_numpy(np.ascontiguousarray(full[top - 1])).cuda()
        got = run_sat(sat, np.ascontiguousarray(a[top:]), carry=carry)
        assert (got == full[top:]).all()
    else:
        b, _ = oracle.sat_f32(a)
        carry = torch.from_numpy(np.ascontiguousarray(b[top - 1].astype(np.float32))).cuda()
        got = run_sat(sat, np.ascontiguousarray(a[top:]), carry=carry)
        # the carry row itself is rounded once to fp32: tolerance of the stacked matrix
        assert_f32_tol(np.concatenate([b[:top].astype(np.float32), got]), a)


# ----------------------------------------------------------------------------------- multi-GPU pieces
@pytest.mark.parametrize("dist", ["u32", "fsym"])
def test_strip_colsum_and_carry_prefix(sat, dist):
    rows, cols = 777, 3001
    a = satgen.gen_host(rows, cols, seed=51, dist=dist)
    _, src = dev_copy(a)
    cs = sat.strip_colsum(src).cpu().numpy()
    if dist == "u32":
        want = oracle.strip_carry_u32(a, cols).view(np.int32)  # column sums of all rows
        assert (cs == want).all()
    else:
        s = oracle.Stream(cols)
        s.rows_f32(a, want_out=False, want_abs=False)
        want = s.colsums_f64()
        assert np.allclose(cs, want, rtol=0, atol=rows * 1.2e-7 * np.abs(a).sum(axis=0).max())
    # carry of rank 2 of 4 = row-wise prefix of (colsum_0 + colsum_1)
    g = np.stack([satgen.gen_host(1, cols, seed=60 + r, dist=dist)[0] for r in range(4)])
    carry = sat.carry_prefix(torch.from_numpy(g).cuda(), 2).cpu().numpy()
    if dist == "u32":
        C = (g[0].view(np.uint32).astype(np.uint64) + g[1].view(np.uint32)) % (1 << 32)
        want = oracle.row_prefix_u32(C.astype(np.uint32)[None, :])[0].view(np.int32)
        assert (carry == want).all()
    else:
        C = g[0].astype(np.float64) + g[1].astype(np.float64)
        want = np.cumsum(C)
        assert np.allclose(carry, want, rtol=0, atol=(cols + 2) * 1.2e-7 * np.cumsum(np.abs(C))[-1])
    assert (sat.carry_prefix(torch.from_numpy(g).cuda(), 0).cpu().numpy() == 0).all()


@pytest.mark.parametrize("nranks", [2, 3, 8])
def test_fake_exchange_sharded_pipeline(sat, nranks):
    """The strip-partition algorithm of sat_compute_sharded on one GPU: the NCCL allgather is replaced by
    stacking the per-strip column sums (everything else is the production path)."""
    rows, cols = 1203, 1777
    a = satgen.gen_host(rows, cols, seed=70 + nranks, dist="u32")
    strips = [sat.strip_bounds(rows, nranks, r) for r in range(nranks)]
    dev = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + n])).cuda() for r0, n in strips]
    gathered = torch.stack([sat.strip_colsum(d) for d in dev])
    outs = []
    for r, d in enumerate(dev):
        carry = sat.carry_prefix(gathered, r)
        outs.append(sat.sat(d, carry=carry) if d.shape[0] else d)
    got = torch.cat(outs).cpu().numpy()
    assert (got == oracle.sat_i32(a)).all()


# ----------------------------------------------------------------------------------- end to end (host buffers)
@pytest.mark.parametrize("dist", ["u32", "fsym"])
def test_host_pipeline(sat, dist):
    rows, cols = 4100, 3000  # > 2 MiB: several pipelined strips
    a = satgen.gen_host(rows, cols, seed=88, dist=dist)
    got = sat.sat_host(a)
    if dist == "u32":
        assert (got == oracle.sat_i32(a)).all()
    else:
        assert_f32_tol(got, a)
    # in place on the host, padded rows: the pad columns must stay untouched
    b = satgen.gen_host(rows, cols, seed=89, dist=dist)
    p = satgen.gen_host(rows, cols, seed=89, dist=dist, pitch=3008)
    p[:, cols:] = 7
    view = p[:, :cols]
    sat.sat_host(view, view)
    assert (p[:, cols:] == 7).all()
    if dist == "u32":
        assert (view == oracle.sat_i32(b)).all()
    else:
        assert_f32_tol(np.ascontiguousarray(view), b)


def test_host_pipeline_concurrent_threads(sat):
    """sat_compute_host from several host threads at once (its per-device staging lock): every
    call's result stays its own.  Sizes differ so that a later call also regrows the staging buffer."""
    import threading

    shapes = [(3000, 2500), (5000, 2100), (1200, 4100), (4100, 3000)]
    inputs = [satgen.gen_host(r, c, seed=700 + k, dist="u32") for k, (r, c) in enumerate(shapes)]
    outs = [None] * len(shapes)
    errs = []

    def run(k):
        try:
            for _ in range(3):
                outs[k] = sat.sat_host(inputs[k])
        except Exception as e:  # pragma: no cover - reported below
            errs.append(e)

    threads = [threading.Thread(target=run, args=(k,)) for k in range(len(shapes))]
    for t in threads:
        t.start()
    for t in threads:
        t.join(timeout=300)
    assert not errs, errs
    for k, a in enumerate(inputs):
        assert (outs[k] == oracle.sat_i32(a)).all(), k


# ----------------------------------------------------------------------------------- tile order (Fig. 9)
@pytest.mark.parametrize("R,C", [(5, 5), (1, 9), (7, 1), (4, 11), (13, 3), (64, 64), (256, 512)])
def test_device_tile_order_matches_fig9_order(sat, R, C):
    got = sat.debug_tile_order(R, C, 0).cpu().numpy()
    want = np.array(oracle.tile_order(R, C))
    assert (got == want).all()
    rm = sat.debug_tile_order(R, C, 1).cpu().numpy()
    assert (rm == np.array([(I, J) for I in range(R) for J in range(C)])).all()


@pytest.mark.parametrize("R,C,g", [(5, 8, 2), (64, 128, 4), (512, 128, 8), (3, 12, 4), (7, 9, 3), (6, 10, 4)])
def test_device_grouped_tile_order_is_topological(sat, R, C, g):
    """Anti-diagonal order of g-wide groups: a permutation of the R x C tiles in which every tile's left,
    upper and upper-left neighbours come first (the look-back's dependencies); with
    g not dividing C the plain Fig. 9 order is used."""
    got = sat.debug_tile_order(R, C, g << 8).cpu().numpy()
    if C % g:
        assert (got == np.array(oracle.tile_order(R, C))).all()
        return
    assert sorted(map(tuple, got.tolist())) == [(I, J) for I in range(R) for J in range(C)]
    pos = {tuple(t): k for k, t in enumerate(got.tolist())}
    for (I, J), k in pos.items():
        for dep in [(I, J - 1), (I - 1, J), (I - 1, J - 1)]:
            if dep[0] >= 0 and dep[1] >= 0:
                assert pos[dep] < k
    assert [tuple(t) for t in got[:g].tolist()] == [(0, j) for j in range(g)]


@pytest.mark.parametrize("R,C,g", [(64, 512, 8), (16, 5, 4), (8, 3, 8), (6, 7, 2), (7, 9, 4), (1, 5, 2)])
def test_device_tall_grouped_tile_order_is_topological(sat, R, C, g):
    """Order 3 (chained strips): anti-diagonal order of g-tall groups, a group's tiles consecutive top to
    bottom; a topological permutation of the R x C tiles; with g not dividing R the
    plain Fig. 9 order."""
    got = sat.debug_tile_order(R, C, 3 | (g << 8)).cpu().numpy()
    if R % g:
        assert (got == np.array(oracle.tile_order(R, C))).all()
        return
    assert sorted(map(tuple, got.tolist())) == [(I, J) for I in range(R) for J in range(C)]
    pos = {tuple(t): k for k, t in enumerate(got.tolist())}
    for (I, J), k in pos.items():
        for dep in [(I, J - 1), (I - 1, J), (I - 1, J - 1)]:
            if dep[0] >= 0 and dep[1] >= 0:
                assert pos[dep] < k
    assert [tuple(t) for t in got[:g].tolist()] == [(i, 0) for i in range(g)]
    # the bottom tile of column J comes R/g group diagonals after the top one
    for J in range(C):
        assert pos[(R - 1, J)] - pos[(0, J)] < (R // g) * (R // g + 1) * g


# ----------------------------------------------------------------------------------- full-size (BASELINE configs)
def _streaming_check(sat, rows, cols, dist, seed, chunk=2048):
    """Full-size parity in the launch configuration bench.py times: device-generated input, one SAT
    launch, then every output row compared with the streaming oracle fed by the host generator."""
    x = torch.empty((rows, cols), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, seed, dist)
    if dist in ("f01", "fsym", "fu2"):
        x = x.view(torch.float32)
    y = sat.sat(x)
    torch.cuda.synchronize()
    del x
    st = oracle.Stream(cols)
    worst = 0.0
    for r0 in range(0, rows, chunk):
        n = min(chunk, rows - r0)
        a = satgen.gen_host(n, cols, seed, dist, row0=r0)
        g = y[r0:r0 + n].cpu().numpy()
        if a.dtype == np.int32:
            want = st.rows_u32(a).view(np.int32)
            if not (g == want).all():
                bad = np.argwhere(g != want)[0]
                raise AssertionError(f"row {r0 + bad[0]} col {bad[1]}: {g[tuple(bad)]} != {want[tuple(bad)]}")
        else:
            want, absw = st.rows_f32(a)
            err = np.abs(g.astype(np.float64) - want)
            tol = oracle.f32_tolerance(absw, rows, cols)
            assert (err <= tol).all(), f"fp32 outside tolerance in rows {r0}..{r0 + n}"
            worst = max(worst, float((err / np.maximum(tol, 1e-300)).max()))
    st.close()
    return worst


@pytest.mark.slow
def test_full_4k_int32_and_fp32(sat):
    _streaming_check(sat, 4096, 4096, "u32", 1447)
    _streaming_check(sat, 4096, 4096, "f01", 1448)


@pytest.mark.slow
def test_full_32k_int32_every_element(sat):
    _streaming_check(sat, 32768, 32768, "u32", 1447)


@pytest.mark.slow
def test_full_32k_fp32_every_element(sat):
    worst = _streaming_check(sat, 32768, 32768, "f01", 1447)
    print(f"32K fp32: worst err/tol = {worst:.3e}")


# ----------------------------------------------------------------------------------------- NCCL path (1 rank)
def _nccl_one_rank(port, q):
    try:
        import os
        import sys
        from pathlib import Path

        sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
        import torch
        import torch.distributed as dist

        import oracle
        import paper_conf_ipps_emotofthni18_b200 as sat
        import satgen

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        torch.cuda.set_device(0)
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
        comm = sat.Comm()
        a = satgen.gen_host(1500, 2100, seed=91, dist="u32")
        x = torch.from_numpy(a).cuda()
        y = sat.sat_sharded(x, comm=comm, check_layout=True)
        torch.cuda.synchronize()
        ok = bool((y.cpu().numpy() == oracle.sat_i32(a)).all())
        comm.close()
        dist.destroy_process_group()
        q.put(("ok" if ok else "mismatch", None))
    except Exception:
        import traceback

        q.put(("error", traceback.format_exc()))


def test_sharded_nccl_single_rank():
    """sat_compute_sharded through a real NCCL communicator (dlopen'ed libnccl, ncclCommInitRank,
    ncclAllGather) with one rank; multi-rank runs need more GPUs than this box has."""
    import socket

    import torch.multiprocessing as mp

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    proc = ctx.Process(target=_nccl_one_rank, args=(port, q))
    proc.start()
    status, err = q.get(timeout=240)
    proc.join(timeout=60)
    assert status == "ok", err


# ----------------------------------------------------------------------------- queries on a SAT
@pytest.mark.parametrize("shape,pitch,rh,rw", [((1, 1), None, 0, 0), ((300, 517), None, 3, 5), ((129, 257), 264, 0, 7),
                                               ((64, 1000), None, 40, 1), ((1009, 203), 208, 12, 12),
                                               ((50, 60), None, 100, 100), ((300, 516), None, 3, 5),
                                               ((40, 3001), 3004, 2, 700), ((33, 2500), None, 1, 1500),
                                               ((20, 5000), None, 25, 0), ((7, 4), None, 0, 3),
                                               # band kernel: many panels / bands, halos across band tops
                                               ((4096, 8192), None, 8, 8), ((2048, 8192), None, 64, 64),
                                               ((3000, 33000), None, 2, 70), ((10000, 300), 304, 50, 3),
                                               ((5000, 1200), None, 0, 0)])
def test_box_sum_int32_bit_exact(sat, shape, pitch, rh, rw):
    b = satgen.gen_host(*shape, seed=31 + shape[0], dist="u32")  # any matrix is a valid operand of P:48
    buf, bd = dev_copy(b, pitch)
    obuf, od = dev_copy(np.zeros_like(b), pitch)
    sat.box_sum(bd, rh, rw, out=od)
    torch.cuda.synchronize()
    got = od.cpu().numpy().view(np.uint32)
    want = oracle.box_sum(b.view(np.uint32), rh, rw)
    assert (got == want).all()
    if pitch is not None and pitch > shape[1]:
        full = obuf[: shape[0] * pitch].view(shape[0], pitch)
        assert (full[:, shape[1]:] == 0x5A5A5A5A).all(), "pad elements were written"


@pytest.mark.parametrize("shape,rh,rw", [((333, 444), 4, 9), ((128, 128), 0, 0), ((1, 2049), 0, 30),
                                         ((65, 2052), 7, 300)])
def test_box_sum_fp32_bit_exact(sat, shape, rh, rw):
    b = satgen.gen_host(*shape, seed=77, dist="fsym")
    _, bd = dev_copy(b)
    got = sat.box_sum(bd, rh, rw).cpu().numpy()
    want = oracle.box_sum(b, rh, rw)  # same fp32 operations in the same order
    assert (got.view(np.uint32) == want.view(np.uint32)).all()


def test_box_filter_end_to_end_from_gpu_sat(sat):
    a = satgen.gen_host(700, 900, seed=5, dist="u32")
    b = sat.sat(torch.from_numpy(a).cuda())
    got = sat.box_sum(b, 6, 11).cpu().numpy().view(np.uint32)
    want = oracle.box_sum(oracle.sat_u32(a), 6, 11)  # oracle SAT, oracle box formula
    assert (got == want).all()
    # spot entries against the direct window sum (the definition)
    for i, j in [(0, 0), (699, 899), (350, 5), (3, 450)]:
        assert int(got[i, j]) == int(a.view(np.uint32)[max(0, i - 6): i + 7, max(0, j - 11): j + 12].astype(np.uint64).sum()) % (1 << 32)


def test_rect_sums_int32_and_fp32(sat):
    rng = np.random.default_rng(9)
    for dist in ("u32", "fsym"):
        b = satgen.gen_host(257, 301, seed=123, dist=dist)
        _, bd = dev_copy(b)
        rows, cols = b.shape
        n = 5000
        r = np.stack([rng.integers(-3, rows + 3, n), rng.integers(-3, rows + 3, n),
                      rng.integers(-3, cols + 3, n), rng.integers(-3, cols + 3, n)], axis=1).astype(np.int64)
        r[:100, 1] = r[:100, 0]  # empty rectangles
        got = sat.rect_sums(bd, torch.from_numpy(r).cuda()).cpu().numpy()
        for k in range(n):
            u = min(max(r[k, 0], -1), rows - 1); d = min(max(r[k, 1], -1), rows - 1)
            l = min(max(r[k, 2], -1), cols - 1); rr = min(max(r[k, 3], -1), cols - 1)
            if u >= d or l >= rr:
                want = 0
            else:
                want = oracle.rect_sum(b.view(np.uint32) if dist == "u32" else b, u, d, l, rr)
            if dist == "u32":
                assert int(got.view(np.uint32)[k]) == int(want), k
            else:
                assert got[k] == np.float32(want), k


def test_query_errors(sat):
    x = torch.zeros((8, 8), dtype=torch.int32, device="cuda")
    with pytest.raises(sat.SatError):
        sat.box_sum(x, -1, 0)
    with pytest.raises(sat.SatError):
        sat.box_sum(x, 1, 1, out=x)


# ----------------------------------------------------------------------------- u8 integral images (NEXT-3)
@pytest.mark.parametrize("shape,spitch,opitch", [((1, 1), None, None), ((300, 517), None, None),
                                                 ((256, 256), 272, 260), ((1000, 2048), None, None),
                                                 ((129, 131), 133, None), ((4096, 4096), None, None),
                                                 ((6000, 6000), None, None), ((777, 3001), 3008, 3004)])
@pytest.mark.parametrize("variant", [-1, 5])  # auto; the flat-tile u8 kernel forced on every shape
def test_u8_integral_image_bit_exact(sat, shape, spitch, opitch, variant):
    rows, cols = shape
    sat.set_tuning(variant, 0, 0)
    a = satgen.gen_host(rows, cols, seed=rows * 7 + cols, dist="u8").astype(np.uint8)
    sp = cols if spitch is None else spitch
    op = cols if opitch is None else opitch
    sbuf = torch.zeros(rows * sp + 64, dtype=torch.uint8, device="cuda")
    src = sbuf[: rows * sp].view(rows, sp)[:, :cols]
    src.copy_(torch.from_numpy(a).cuda())
    obuf = torch.full((rows * op + 64,), 0x5A5A5A5A, dtype=torch.int32, device="cuda")
    out = obuf[: rows * op].view(rows, op)[:, :cols]
    try:
        sat.sat_u8(src, out=out)
        torch.cuda.synchronize()
    finally:
        sat.set_tuning(-1, 0, 0)
    got = out.cpu().numpy().view(np.uint32)
    want = oracle.sat_u32(a.astype(np.uint32))
    assert (got == want).all()
    if op > cols:
        assert (obuf[: rows * op].view(rows, op)[:, cols:] == 0x5A5A5A5A).all(), "pad elements were written"


def test_u8_full_32k_sampled_rows(sat):
    n = 32768
    t = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(t, 1451, "u8")
    a = t.to(torch.uint8)
    del t
    b = sat.sat_u8(a)
    torch.cuda.synchronize()
    st = oracle.Stream(n)
    check_rows = {0, 1, 127, 128, 4095, 20000, n - 1}
    for i0 in range(0, n, 2048):
        rows = st.rows_u32(a[i0: i0 + 2048].cpu().numpy().astype(np.uint32))
        for i in check_rows:
            if i0 <= i < i0 + 2048:
                assert (b[i].cpu().numpy().view(np.uint32) == rows[i - i0]).all(), i
