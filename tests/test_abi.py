"""The C-ABI library loads and exports every symbol include/sat.h declares; host-side argument
handling that needs no GPU.  CPU only: no compute call reaches a kernel here."""
import ctypes
import re
from pathlib import Path

import pytest

ROOT = Path(__file__).resolve().parent.parent
HEADER = ROOT / "include" / "sat.h"


@pytest.fixture(scope="module")
def sat():
    import build_native

    build_native.build_libsat()
    import paper_conf_ipps_emotofthni18_b200 as sat

    return sat


def declared_symbols():
    text = HEADER.read_text()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(sat_[a-z0-9_]+)\s*\(", text)))


def test_header_declares_the_north_star_entry_points():
    names = declared_symbols()
    for must in ("sat_compute_i32", "sat_compute_f32", "sat_compute_sharded"):
        assert must in names


def test_library_exports_every_declared_symbol(sat):
    lib = ctypes.CDLL(str(ROOT / "paper_conf_ipps_emotofthni18_b200" / "libsat.so"))
    for name in declared_symbols():
        assert hasattr(lib, name), f"libsat.so does not export {name}"
    from paper_conf_ipps_emotofthni18_b200 import _lib

    assert sorted(_lib.EXPORTS) == declared_symbols()


def test_version_and_status_strings(sat):
    from paper_conf_ipps_emotofthni18_b200 import _lib

    assert sat.version() == 100
    for code, name in _lib.STATUS_NAMES.items():
        assert _lib.lib().sat_status_string(code).decode() == name


def test_variants_and_tuning(sat):
    n = sat.num_variants()
    assert n >= 1
    shapes = [sat.variant_info(v) for v in range(n)]
    # tiles of 64 KiB or less, 128 columns per lane chunk (flat 64 x 256 tiles are the production shape)
    assert all(tc % 128 == 0 and tr % 32 == 0 and tr * tc <= 128 * 128 for tr, tc in shapes)
    assert (64, 256) in shapes and (128, 128) in shapes
    with pytest.raises(sat.SatError):
        sat.variant_info(n)
    with pytest.raises(sat.SatError):
        sat.set_tuning(n, 0, 0)
    with pytest.raises(sat.SatError):
        sat.set_tuning(-1, 4, 0)
    sat.set_tuning(-1, 3 | (8 << 8), 0)  # anti-diagonal order of 8-tall tile groups (chained strips)
    with pytest.raises(sat.SatError):
        sat.set_tuning(-1, 0x201 | 0x10000, 0)
    sat.set_tuning(-1, 0x200, 0)  # anti-diagonal order of 2-tile groups
    sat.set_tuning(-1, 0, 0)
    sat.set_max_ctas(0)


def test_argument_validation_without_gpu(sat):
    from paper_conf_ipps_emotofthni18_b200 import _lib

    L = _lib.lib()
    # empty problems are no-ops (no CUDA call needed)
    assert L.sat_compute(0, None, None, 0, 5, 5, None, None) == 0
    assert L.sat_compute(1, None, None, 7, 0, 0, None, None) == 0
    # bad sizes are rejected before any CUDA call
    assert L.sat_compute(0, 16, 16, 4, 8, 7, None, None) == 1  # pitch < cols
    assert L.sat_compute(0, 16, 16, -1, 8, 8, None, None) == 1
    assert L.sat_compute(7, 16, 16, 4, 8, 8, None, None) == 1  # unknown dtype
    assert L.sat_compute(0, 18, 1 << 20, 4, 8, 8, None, None) == 2  # misaligned
    assert L.sat_compute(0, 1 << 20, (1 << 20) + 16, 4, 8, 8, None, None) == 1  # partial overlap
    assert b"overlap" in L.sat_last_error_detail()
    assert L.sat_compute_host(0, None, None, 3, 4, 2, None) == 1


def test_plan_shapes(sat):
    p = sat.query_plan(sat.SAT_INT32, 1000, 1000, 1024, 1 << 20, 1 << 21)
    tr, tc = p["tile_rows"], p["tile_cols"]
    assert p["tiles"] == -(-1000 // tr) * -(-1000 // tc)
    assert p["tma"] == 1
    assert p["aux_bytes"] == p["tiles"] * (tr + tc + 1) * 8
    assert sat.query_plan(sat.SAT_INT32, 1000, 1000, 1001, 1 << 20, 1 << 21)["tma"] == 0  # pitch*4 % 16
    assert sat.query_plan(sat.SAT_INT32, 10, 10, 12, (1 << 20) + 4, 1 << 21)["tma"] == 0  # pointer % 16


def test_strip_bounds_cover_rows_exactly(sat):
    for rows in [0, 1, 7, 64, 65536, 65537]:
        for world in [1, 2, 3, 8]:
            parts = [sat.strip_bounds(rows, world, r) for r in range(world)]
            assert sum(n for _, n in parts) == rows
            pos = 0
            for r0, n in parts:
                assert n >= 0 and (n == 0 or r0 == pos)
                pos += n


def test_batched_argument_validation_without_gpu(sat):
    """sat_compute_batched / _u8 reject bad arguments before any CUDA call (include/sat.h)."""
    from paper_conf_ipps_emotofthni18_b200 import _lib

    L = _lib.lib()
    B = L.sat_compute_batched
    assert B(0, None, None, 0, 5, 5, 5, 25, None) == 0  # empty batch: no-op, null pointers allowed
    assert B(1, None, None, 3, 0, 5, 5, 25, None) == 0  # empty matrices
    assert B(0, 16, 16, -1, 4, 8, 8, 32, None) == 1  # negative batch
    assert B(0, 16, 16, 2, 4, 8, 7, 32, None) == 1  # pitch < cols
    assert B(5, 16, 16, 2, 4, 8, 8, 32, None) == 1  # unknown dtype
    assert B(0, 16, 16, 2, 4, 8, 8, 31, None) == 1  # image stride < (rows-1)*pitch + cols
    assert b"overlap" in L.sat_last_error_detail()
    assert B(0, 18, 1 << 20, 2, 4, 8, 8, 32, None) == 2  # misaligned
    assert B(0, 1 << 20, (1 << 20) + 64, 2, 4, 8, 8, 32, None) == 1  # batches partially overlap
    U = L.sat_compute_batched_u8
    assert U(None, 8, 32, None, 0, 4, 8, 8, 32, None) == 0
    assert U(16, 7, 32, 1 << 20, 2, 4, 8, 8, 32, None) == 1  # src_pitch < cols
    assert U(16, 8, 31, 1 << 20, 2, 4, 8, 8, 32, None) == 1  # src image stride too small
    assert U(16, 8, 32, (1 << 20) + 2, 2, 4, 8, 8, 32, None) == 2  # dst misaligned
    assert U(1 << 20, 8, 32, (1 << 20) + 8, 2, 4, 8, 8, 32, None) == 1  # src and dst overlap


def test_batched_binding_rejects_bad_tensors(sat):
    torch = pytest.importorskip("torch")
    with pytest.raises(ValueError):
        sat.sat_batched(torch.zeros(2, 3, 4, dtype=torch.int32))  # not a CUDA tensor
    with pytest.raises(ValueError):
        sat.sat_batched_u8(torch.zeros(2, 3, 4, dtype=torch.uint8))


def test_wide_argument_validation_without_gpu(sat):
    """sat_compute_f32_f64 / sat_compute_moments_f32 reject bad arguments before any CUDA call."""
    from paper_conf_ipps_emotofthni18_b200 import _lib

    L = _lib.lib()
    for F in (L.sat_compute_f32_f64, L.sat_compute_moments_f32):
        assert F(None, 5, None, 5, 0, 5, None) == 0  # empty: no-op, null pointers allowed
        assert F(None, 5, None, 5, 4, 0, None) == 0
        assert F(1 << 20, 4, 1 << 21, 5, 4, 5, None) == 1  # src_pitch < cols
        assert F(1 << 20, 5, 1 << 21, 4, 4, 5, None) == 1  # dst_pitch < cols
        assert F(1 << 20, 5, 1 << 21, 5, -1, 5, None) == 1  # negative rows
        assert F(None, 5, 1 << 21, 5, 4, 5, None) == 1  # null src
        assert F((1 << 20) + 2, 5, 1 << 21, 5, 4, 5, None) == 2  # src not 4-byte aligned
        assert F(1 << 20, 5, (1 << 21) + 4, 5, 4, 5, None) == 2  # dst not 8-byte aligned
        assert F(1 << 20, 5, (1 << 20) + 8, 5, 4, 5, None) == 1  # overlap
        assert b"overlap" in L.sat_last_error_detail()
