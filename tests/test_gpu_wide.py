"""64-bit-element SATs against the CPU oracle, through the C ABI:

* sat_compute_f32_f64 (sat.sat_f64): fp32 in, fp64 SAT out -- oracle.sat_f32 (column-then-row P:46 in
  fp64); tolerance (rows + cols) * 2.3e-16 * absSAT (reading R10 with the fp64 unit roundoff), bit-exact
  in the integer regime;
* sat_compute_moments_f32 (sat.sat_moments): (SAT(a), SAT(a*a)) fp32 pairs (ref. [8] P:311) --
  oracle.moments_f32; each channel within (rows + cols) * 1.2e-7 * its absSAT, bit-exact in the integer
  regime (a in {0..3}, every partial sum < 2^24).
Needs a B200."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

SHAPES = [(1, 1), (1, 300), (300, 1), (64, 128), (65, 129), (300, 517), (1000, 3000), (2048, 2048), (129, 4099)]


@pytest.fixture(scope="module")
def sat():
    import paper_conf_ipps_emotofthni18_b200 as sat

    return sat


def f64_tol(ab, rows, cols):
    return (rows + cols) * 2.3e-16 * ab


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("dist", ["fsym", "f01"])
def test_f64_within_tolerance(sat, shape, dist):
    a = satgen.gen_host(*shape, seed=3100 + shape[0], dist=dist)
    got = sat.sat_f64(torch.from_numpy(a).cuda()).cpu().numpy()
    b, ab = oracle.sat_f32(a)
    assert got.dtype == np.float64
    assert (np.abs(got - b) <= f64_tol(ab, *shape)).all()


@pytest.mark.parametrize("shape", [(300, 517), (2048, 2048), (4096, 4096)])
def test_f64_integer_regime_bit_exact(sat, shape):
    a = satgen.gen_host(*shape, seed=3200, dist="fu2")
    got = sat.sat_f64(torch.from_numpy(a).cuda()).cpu().numpy()
    b, _ = oracle.sat_f32(a)
    assert (got == b).all()


def test_f64_beats_fp32_where_fp32_rounds(sat):
    """4K x 4K of U[0,1): the fp64 path stays within its fp64 bound where the fp32 SAT needs the fp32 one."""
    n = 4096
    a = satgen.gen_host(n, n, seed=3300, dist="f01")
    x = torch.from_numpy(a).cuda()
    b, ab = oracle.sat_f32(a)
    got64 = sat.sat_f64(x).cpu().numpy()
    got32 = sat.sat(x).cpu().numpy().astype(np.float64)
    e64, e32 = np.abs(got64 - b).max(), np.abs(got32 - b).max()
    assert (np.abs(got64 - b) <= f64_tol(ab, n, n)).all()
    assert e64 < e32 * 1e-6


def test_f64_pitched_layouts_and_pads(sat):
    rows, cols = 333, 700
    a = satgen.gen_host(rows, cols, seed=3400, dist="fsym")
    src = torch.zeros((rows, 705), dtype=torch.float32, device="cuda")
    src[:, :cols] = torch.from_numpy(a).cuda()
    out = torch.full((rows, 703), 7.0, dtype=torch.float64, device="cuda")
    sat.sat_f64(src[:, :cols], out=out[:, :cols])
    b, ab = oracle.sat_f32(a)
    o = out.cpu().numpy()
    assert (np.abs(o[:, :cols] - b) <= f64_tol(ab, rows, cols)).all()
    assert (o[:, cols:] == 7.0).all()  # pad columns never written


def test_f64_repeated_calls_one_stream(sat):
    a = satgen.gen_host(1500, 1700, seed=3500, dist="fu2")
    x = torch.from_numpy(a).cuda()
    b, _ = oracle.sat_f32(a)
    for _ in range(20):  # epochs advance per launch; no workspace reset
        assert (sat.sat_f64(x).cpu().numpy() == b).all()


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("dist", ["fsym", "f01"])
def test_moments_within_tolerance(sat, shape, dist):
    a = satgen.gen_host(*shape, seed=3600 + shape[1], dist=dist)
    got = sat.sat_moments(torch.from_numpy(a).cuda()).cpu().numpy().astype(np.float64)
    s1, ab1, s2, ab2 = oracle.moments_f32(a)
    rows, cols = shape
    assert (np.abs(got[..., 0] - s1) <= (rows + cols) * 1.2e-7 * ab1).all()
    assert (np.abs(got[..., 1] - s2) <= (rows + cols) * 1.2e-7 * ab2).all()


@pytest.mark.parametrize("shape", [(300, 517), (1024, 1024)])
def test_moments_integer_regime_bit_exact(sat, shape):
    a = satgen.gen_host(*shape, seed=3700, dist="fu2")
    got = sat.sat_moments(torch.from_numpy(a).cuda()).cpu().numpy().astype(np.float64)
    s1, _, s2, _ = oracle.moments_f32(a)
    assert (got[..., 0] == s1).all() and (got[..., 1] == s2).all()


def test_moments_variance_of_a_box(sat):
    """The SAVSM use (P:48-50 applied to both channels): mean and variance of a window from 4 reads each."""
    a = satgen.gen_host(200, 300, seed=3800, dist="fu2")
    m = sat.sat_moments(torch.from_numpy(a).cuda()).cpu().numpy().astype(np.float64)
    u, d, l, r = 40, 90, 100, 180  # rows u+1..d, cols l+1..r
    n = (d - u) * (r - l)
    s = m[d, r] - m[u, r] - m[d, l] + m[u, l]
    w = a[u + 1:d + 1, l + 1:r + 1].astype(np.float64)
    assert s[0] == w.sum() and s[1] == (w * w).sum()
    assert abs((s[1] / n - (s[0] / n) ** 2) - w.var()) < 1e-9


def test_wide_argument_errors(sat):
    x = torch.zeros((10, 20), dtype=torch.float32, device="cuda")
    with pytest.raises(TypeError):
        sat.sat_f64(x.to(torch.float64))
    with pytest.raises(ValueError):
        sat.sat_f64(x, out=torch.zeros((10, 20), dtype=torch.float32, device="cuda"))
    with pytest.raises(ValueError):
        sat.sat_moments(x, out=torch.zeros((10, 20, 3), dtype=torch.float32, device="cuda"))
    buf = torch.zeros(4096, dtype=torch.float64, device="cuda")
    with pytest.raises(sat.SatError):  # dst overlapping src
        lib = sat._lib.lib()
        sat._lib.check(lib.sat_compute_f32_f64(buf.data_ptr(), 20, buf.data_ptr() + 8, 20, 10, 20, None), "f64")
    with pytest.raises(sat.SatError):  # misaligned dst
        sat._lib.check(lib.sat_compute_f32_f64(x.data_ptr(), 20, buf.data_ptr() + 4, 20, 10, 20, None), "f64")
    sat._lib.check(lib.sat_compute_f32_f64(x.data_ptr(), 20, buf.data_ptr(), 20, 0, 20, None), "f64")  # no-op
