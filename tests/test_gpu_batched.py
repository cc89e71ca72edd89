"""GPU parity of sat_compute_batched (SATs of a batch of small matrices in one launch, SURVEY.md
Sec. 8(f) NEXT-2) against the CPU oracle, matrix by matrix on the same seeded inputs: int32
bit-exact (uint32 wraparound), fp32 within (rows+cols) * 1.2e-7 * absSAT and bit-exact in the exact
regime (inputs in {0..3}).  Shapes span the four CTA widths (1/2/4/8 warps per row chunk), images
wider than one 1024-column chunk, ragged bands and columns, row/image padding, in place, and the
scalar (unaligned) path.  Needs a B200."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

SENTINEL = 0x5A5A5A5A


@pytest.fixture(scope="module")
def sat():
    import paper_conf_ipps_emotofthni18_b200 as sat

    return sat


def make_batch(batch, rows, cols, dist, seed):
    # image k = rows [k*rows, (k+1)*rows) of one seeded matrix (the generator is counter-based)
    a = satgen.gen_host(batch * rows, cols, seed, dist)
    return a.reshape(batch, rows, cols)


def upload(a, pitch, stride, offset_words=0):
    """Device buffer holding the batch with row stride `pitch` and image stride `stride` (elements);
    every other word is the sentinel.  Returns (buffer, strided 3-D view)."""
    batch, rows, cols = a.shape
    n = (batch - 1) * stride + (rows - 1) * pitch + cols
    buf = torch.full((n + offset_words + 16,), SENTINEL, dtype=torch.int32, device="cuda")
    view = torch.as_strided(buf, (batch, rows, cols), (stride, pitch, 1), offset_words)
    view.copy_(torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).to("cuda"))
    if a.dtype == np.float32:
        view = view.view(torch.float32)
    return buf, view


def check_images(got, a):
    for k in range(a.shape[0]):
        if a.dtype == np.float32:
            b, ab = oracle.sat_f32(a[k])
            tol = oracle.f32_tolerance(ab, *a.shape[1:])
            err = np.abs(got[k].astype(np.float64) - b)
            assert (err <= tol).all(), f"image {k}: fp32 outside tolerance, max excess {np.max(err - tol)}"
        else:
            want = oracle.sat_i32(a[k])
            bad = np.argwhere(got[k].view(np.int32) != want)
            assert len(bad) == 0, f"image {k}: {len(bad)} mismatches, first at {bad[0].tolist()}"


def run(sat, a, pitch=None, stride=None, inplace=False, offset_words=0):
    batch, rows, cols = a.shape
    pitch = cols if pitch is None else pitch
    stride = rows * pitch if stride is None else stride
    buf, src = upload(a, pitch, stride, offset_words)
    if inplace:
        obuf, out = buf, src
    else:
        obuf, out = upload(np.zeros_like(a), pitch, stride, offset_words)
    sat.sat_batched(src, out=out)
    torch.cuda.synchronize()
    got = out.cpu().numpy()
    # words outside the matrices (row pads, image pads, guard words) are never written
    mask = torch.ones_like(obuf, dtype=torch.bool)
    torch.as_strided(mask, (batch, rows, cols), (stride, pitch, 1), offset_words).fill_(False)
    outside = obuf[mask]
    if not inplace:
        assert (outside == SENTINEL).all(), "words outside the matrices were written"
    return got


@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 9, 9), (5, 1, 700), (4, 700, 1), (7, 33, 100), (6, 64, 128),
                                   (5, 65, 129), (9, 100, 256), (4, 129, 257), (3, 256, 512), (3, 250, 513),
                                   (2, 300, 1024), (2, 77, 1025), (2, 40, 2500)])
@pytest.mark.parametrize("dist", ["u32", "f01", "fsym"])
def test_batched_parity(sat, shape, dist):
    a = make_batch(*shape, dist=dist, seed=4242 + shape[1] * 7 + shape[2])
    check_images(run(sat, a), a)


def test_batched_exact_regime_f32(sat):
    # inputs in {0..3}: every partial sum is an integer < 2^24, so fp32 is bit-exact
    a = make_batch(6, 200, 300, dist="fu2", seed=7)
    got = run(sat, a)
    for k in range(a.shape[0]):
        want = oracle.sat_i32(a[k].astype(np.int32))
        assert (got[k].astype(np.int64) == want).all()


@pytest.mark.parametrize("pitch,stride,offset", [(132, None, 0), (131, None, 1), (128, 128 * 50 + 4, 0),
                                                 (130, 130 * 50 + 3, 2)])
def test_batched_pitch_stride(sat, pitch, stride, offset):
    # padded rows / images and misaligned bases take the scalar path when not 16-byte aligned
    a = make_batch(5, 50, 127, dist="u32", seed=31)
    check_images(run(sat, a, pitch=pitch, stride=stride, offset_words=offset), a)


@pytest.mark.parametrize("dist", ["u32", "fsym"])
def test_batched_inplace(sat, dist):
    a = make_batch(4, 90, 2100, dist=dist, seed=5)  # three column chunks: left terms read back in place
    check_images(run(sat, a, inplace=True), a)


def test_batched_many_images(sat):
    # more images than the launch's CTA cap (148 x 64): the CTAs loop over images
    a = make_batch(148 * 64 + 37, 4, 16, dist="u32", seed=11)
    got = run(sat, a)
    want = np.stack([oracle.sat_i32(a[k]) for k in range(0, a.shape[0], 997)])
    assert (got[::997].view(np.int32) == want).all()
    totals = a.view(np.uint32).sum(axis=(1, 2), dtype=np.uint64).astype(np.uint32)
    assert (got[:, -1, -1].astype(np.uint32) == totals).all()


def test_batched_matches_single(sat):
    # the batched and single-matrix paths agree bit-exactly for int32
    a = make_batch(3, 513, 777, dist="u32", seed=3)
    got = run(sat, a)
    for k in range(3):
        t = torch.from_numpy(a[k].copy()).cuda()
        assert (sat.sat(t).cpu().numpy() == got[k]).all()


def test_batched_edge_cases(sat):
    t = torch.zeros((0, 5, 5), dtype=torch.int32, device="cuda")
    sat.sat_batched(t)  # empty batch: no-op
    t = torch.zeros((3, 0, 5), dtype=torch.int32, device="cuda")
    sat.sat_batched(t)
    lib = sat._lib.lib()
    x = torch.zeros(1024, dtype=torch.int32, device="cuda")
    # overlapping images (stride < span) are rejected
    assert lib.sat_compute_batched(0, x.data_ptr(), x.data_ptr(), 2, 4, 8, 8, 16, None) == 1
    # partial overlap of src and dst
    assert lib.sat_compute_batched(0, x.data_ptr(), x.data_ptr() + 16, 2, 4, 8, 8, 32, None) == 1
    # misaligned pointer
    assert lib.sat_compute_batched(0, x.data_ptr() + 2, x.data_ptr() + 2048, 1, 4, 8, 8, 32, None) == 2
    # negative batch, pitch < cols, bad dtype
    assert lib.sat_compute_batched(0, x.data_ptr(), x.data_ptr(), -1, 4, 8, 8, 32, None) == 1
    assert lib.sat_compute_batched(0, x.data_ptr(), x.data_ptr(), 1, 4, 8, 7, 32, None) == 1
    assert lib.sat_compute_batched(9, x.data_ptr(), x.data_ptr(), 1, 4, 8, 8, 32, None) == 1


# ---------------------------------------------------------------- u8 images -> uint32 integral images

def make_u8(batch, rows, cols, seed):
    return make_batch(batch, rows, cols, dist="u8", seed=seed).astype(np.uint8)


def run_u8(sat, img, spitch=None, sstride=None, soff=0, pitch=None, stride=None):
    batch, rows, cols = img.shape
    spitch = cols if spitch is None else spitch
    sstride = rows * spitch if sstride is None else sstride
    pitch = cols if pitch is None else pitch
    stride = rows * pitch if stride is None else stride
    n = (batch - 1) * sstride + (rows - 1) * spitch + cols
    sbuf = torch.full((n + soff + 16,), 0xA5, dtype=torch.uint8, device="cuda")
    src = torch.as_strided(sbuf, (batch, rows, cols), (sstride, spitch, 1), soff)
    src.copy_(torch.from_numpy(np.ascontiguousarray(img)).cuda())
    m = (batch - 1) * stride + (rows - 1) * pitch + cols
    obuf = torch.full((m + 16,), SENTINEL, dtype=torch.int32, device="cuda")
    out = torch.as_strided(obuf, (batch, rows, cols), (stride, pitch, 1))
    sat.sat_batched_u8(src, out=out)
    torch.cuda.synchronize()
    mask = torch.ones_like(obuf, dtype=torch.bool)
    torch.as_strided(mask, (batch, rows, cols), (stride, pitch, 1)).fill_(False)
    assert (obuf[mask] == SENTINEL).all(), "words outside the integral images were written"
    return out.cpu().numpy()


@pytest.mark.parametrize("shape", [(1, 1, 1), (5, 9, 9), (4, 100, 128), (3, 65, 129), (3, 200, 256),
                                   (2, 129, 513), (2, 300, 1024), (2, 50, 2047)])
def test_batched_u8_parity(sat, shape):
    img = make_u8(*shape, seed=900 + shape[2])
    got = run_u8(sat, img)
    for k in range(shape[0]):
        assert (got[k] == oracle.sat_i32(img[k].astype(np.int32))).all(), f"image {k}"


@pytest.mark.parametrize("spitch,sstride,soff,pitch", [(130, None, 0, None), (128, 128 * 40 + 4, 0, 132),
                                                       (128, None, 1, None), (131, 131 * 40 + 5, 3, 129)])
def test_batched_u8_layouts(sat, spitch, sstride, soff, pitch):
    img = make_u8(4, 40, 127, seed=17)
    got = run_u8(sat, img, spitch=spitch, sstride=sstride, soff=soff, pitch=pitch)
    for k in range(4):
        assert (got[k] == oracle.sat_i32(img[k].astype(np.int32))).all()


def test_batched_u8_wraps_mod_2_32(sat):
    # all-255 images whose totals pass 2^31 and 2^32: the uint32 bit pattern (mod 2^32)
    img = np.full((2, 3000, 6000), 255, dtype=np.uint8)
    got = run_u8(sat, img)
    i, j = np.arange(3000)[:, None] + 1, np.arange(6000)[None, :] + 1
    want = ((i * j * 255) % (1 << 32)).astype(np.uint32).view(np.int32)
    assert (got[0] == want).all() and (got[1] == want).all()


def test_batched_u8_matches_single(sat):
    img = make_u8(3, 333, 1500, seed=23)
    got = run_u8(sat, img)
    for k in range(3):
        assert (sat.sat_u8(torch.from_numpy(img[k].copy()).cuda()).cpu().numpy() == got[k]).all()


def test_sat_calls_replay_from_a_cuda_graph():
    """Small matrices are launch-latency bound (NEXT-2): after one warm-up call on a stream (which
    creates that stream's workspace), sat_compute is capturable -- epochs advance on the device, no host
    sync -- so a CUDA graph of many calls replays with exact results every time."""
    import paper_conf_ipps_emotofthni18_b200 as sat

    shapes = [(256, 256), (300, 517), (1024, 1024), (64, 2000)]
    xs = [torch.from_numpy(satgen.gen_host(r, c, seed=900 + r, dist="u32")).cuda() for r, c in shapes]
    ys = [torch.empty_like(x) for x in xs]
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for x, y in zip(xs, ys):
            sat.sat(x, out=y, stream=s)  # warm-up: workspace, occupancy caches
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(3):
            for x, y in zip(xs, ys):
                sat.sat(x, out=y, stream=s)
    for _ in range(5):
        for y in ys:
            y.zero_()
        g.replay()
        torch.cuda.synchronize()
        for x, y in zip(xs, ys):
            assert (y.cpu().numpy() == oracle.sat_i32(x.cpu().numpy())).all()
