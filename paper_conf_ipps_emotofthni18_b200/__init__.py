"""libsat Python binding: single-pass summed area tables on B200 (sm_100a).

Thin marshalling over the C ABI of include/sat.h (same names).  Every step of the computation runs
in libsat's CUDA kernels; PyTorch supplies device memory, streams and process groups only.  There
is no CPU fallback: importing this package without a built libsat.so raises ImportError.

    import paper_conf_ipps_emotofthni18_b200 as sat
    b = sat.sat(a)                       # a: 2-D int32/float32 CUDA tensor (row stride = pitch)
    sat.sat(a, out=a)                    # in place
    sat.sat_host(np_array)               # host buffers -> host result (H2D + SAT + D2H pipeline)
    comm = sat.Comm(group)               # NCCL communicator over a torch process group
    sat.sat_sharded(strip, comm=comm)    # strip-partitioned SAT across ranks
"""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import SAT_FLOAT32, SAT_INT32, SatError, SatPlan, check

_lib.lib()  # load now: fail loudly at import if the native library is missing

__all__ = [
    "sat", "sat_batched", "sat_batched_u8", "sat_u8", "sat_f64", "sat_moments", "sat_host", "compute", "box_sum", "rect_sums", "strip_colsum", "carry_prefix", "Comm", "sat_sharded", "strip_bounds",
    "Chain", "sat_chained", "exchange_blobs",
    "strip_layout", "broadcast_unique_id",
    "query_plan", "set_tuning", "set_max_ctas", "num_variants", "variant_info", "debug_tile_order", "debug_occupy", "debug_workspace",
    "release_stream_workspace", "release_workspaces",
    "version", "SatError", "SAT_INT32", "SAT_FLOAT32",
]


def _torch():
    import torch

    return torch


def _dtype_code(t) -> int:
    torch = _torch()
    if t.dtype == torch.int32:
        return SAT_INT32
    if t.dtype == torch.float32:
        return SAT_FLOAT32
    raise TypeError(f"libsat supports int32 and float32, got {t.dtype}")


def _stream_ptr(stream) -> int:
    torch = _torch()
    s = torch.cuda.current_stream() if stream is None else stream
    return int(s.cuda_stream)


def _check_vec_out(out, n: int, dtype, device, name: str = "out"):
    """A caller-supplied output vector: contiguous, `n` elements of `dtype` on `device`."""
    if out.dtype != dtype or out.numel() != n or not out.is_contiguous() or out.device != device:
        raise ValueError(f"{name} must be a contiguous tensor of {n} elements, dtype {dtype}, on {device}")


def _matrix(t, name: str):
    if not t.is_cuda or t.dim() != 2 or t.stride(1) != 1 or (t.shape[0] > 1 and t.stride(0) < t.shape[1]):
        raise ValueError(f"{name}: need a 2-D CUDA tensor with unit column stride and row stride >= cols")
    return t.shape[0], t.shape[1], (t.stride(0) if t.shape[0] > 1 else max(t.stride(0), t.shape[1]))


def compute(dtype: int, src_ptr: int, dst_ptr: int, rows: int, cols: int, pitch: int, carry_ptr: int = 0,
            stream_ptr: int = 0) -> None:
    """Raw C-ABI call sat_compute (device pointers)."""
    check(_lib.lib().sat_compute(dtype, src_ptr, dst_ptr, rows, cols, pitch, carry_ptr or None, stream_ptr or None),
          "sat_compute")


def sat(src, out=None, *, carry=None, stream=None):
    """SAT of a 2-D int32/float32 CUDA tensor.  ``out`` may be ``src`` (in place) or a tensor of
    the same shape and row stride; ``carry`` (1-D, cols) is added to every row of the result."""
    torch = _torch()
    rows, cols, pitch = _matrix(src, "src")
    if out is None:
        out = torch.empty_strided((rows, cols), (pitch, 1), dtype=src.dtype, device=src.device)
    orows, ocols, opitch = _matrix(out, "out")
    if (orows, ocols, opitch) != (rows, cols, pitch) or out.dtype != src.dtype or out.device != src.device:
        raise ValueError("out must match src in shape, row stride, dtype and device")
    cptr = 0
    if carry is not None:
        if carry.dtype != src.dtype or carry.numel() != cols or not carry.is_contiguous() or carry.device != src.device:
            raise ValueError("carry must be a contiguous vector of `cols` elements of src's dtype and device")
        cptr = carry.data_ptr()
    with torch.cuda.device(src.device):
        compute(_dtype_code(src), src.data_ptr(), out.data_ptr(), rows, cols, pitch, cptr, _stream_ptr(stream))
    return out


def sat_batched(src, out=None, *, stream=None):
    """SATs of a batch of matrices (P:44 per matrix) in one launch: ``src`` is a 3-D int32/float32
    CUDA tensor (batch, rows, cols) with unit column stride; ``out`` may be ``src`` (in place) or a
    tensor of the same shape and strides.  For many small matrices."""
    torch = _torch()
    if not src.is_cuda or src.dim() != 3 or src.stride(2) != 1:
        raise ValueError("src: need a 3-D CUDA tensor (batch, rows, cols) with unit column stride")
    batch, rows, cols = src.shape
    pitch = src.stride(1) if rows > 1 else max(src.stride(1), cols)
    stride = src.stride(0) if batch > 1 else max(src.stride(0), (rows - 1) * pitch + cols)
    if out is None:
        out = torch.empty_strided(tuple(src.shape), src.stride(), dtype=src.dtype, device=src.device)
    if out.shape != src.shape or out.stride() != src.stride() or out.dtype != src.dtype or out.device != src.device:
        raise ValueError("out must match src in shape, strides, dtype and device")
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_compute_batched(_dtype_code(src), src.data_ptr(), out.data_ptr(), batch, rows, cols,
                                             pitch, stride, _stream_ptr(stream)), "sat_compute_batched")
    return out


def sat_batched_u8(src, out=None, *, stream=None):
    """Integral images of a batch of uint8 images: ``src`` is a 3-D uint8 CUDA tensor (batch, rows, cols)
    with unit column stride; returns an int32 tensor of the same shape holding the uint32 SATs."""
    torch = _torch()
    if src.dtype != torch.uint8 or not src.is_cuda or src.dim() != 3 or src.stride(2) != 1:
        raise ValueError("src: need a 3-D uint8 CUDA tensor (batch, rows, cols) with unit column stride")
    batch, rows, cols = src.shape
    spitch = src.stride(1) if rows > 1 else max(src.stride(1), cols)
    sstride = src.stride(0) if batch > 1 else max(src.stride(0), (rows - 1) * spitch + cols)
    if out is None:
        out = torch.empty((batch, rows, cols), dtype=torch.int32, device=src.device)
    if out.dtype != torch.int32 or out.device != src.device or out.shape != src.shape or out.stride(2) != 1:
        raise ValueError("out must be an int32 tensor of src's shape on src's device, unit column stride")
    pitch = out.stride(1) if rows > 1 else max(out.stride(1), cols)
    stride = out.stride(0) if batch > 1 else max(out.stride(0), (rows - 1) * pitch + cols)
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_compute_batched_u8(src.data_ptr(), spitch, sstride, out.data_ptr(), batch, rows, cols,
                                                pitch, stride, _stream_ptr(stream)), "sat_compute_batched_u8")
    return out


def sat_host(src, out=None, *, stream=None):
    """End-to-end C-ABI call with host buffers (numpy int32/float32 2-D arrays, or CPU torch tensors).
    Copies in, computes, copies out; synchronous.  Returns ``out``."""
    import numpy as np

    torch = _torch()
    arr = src.numpy() if hasattr(src, "numpy") and not isinstance(src, np.ndarray) else src
    if arr.ndim != 2 or arr.dtype not in (np.int32, np.float32) or arr.strides[1] != 4:
        raise ValueError("src must be a 2-D int32/float32 host array with unit column stride")
    if out is None:
        out = np.empty_like(arr)
    oarr = out.numpy() if hasattr(out, "numpy") and not isinstance(out, np.ndarray) else out
    if oarr.shape != arr.shape or oarr.dtype != arr.dtype or oarr.strides != arr.strides:
        raise ValueError("out must match src in shape, dtype and strides")
    rows, cols = arr.shape
    pitch = arr.strides[0] // 4 if rows > 1 else cols
    code = SAT_INT32 if arr.dtype == np.int32 else SAT_FLOAT32
    check(_lib.lib().sat_compute_host(code, arr.ctypes.data, oarr.ctypes.data, rows, cols, pitch,
                                      _stream_ptr(stream) if torch.cuda.is_available() else None),
          "sat_compute_host")
    return out


def sat_u8(src, out=None, *, stream=None):
    """Integral image of a 2-D uint8 CUDA tensor: uint32 SAT returned as an int32 tensor holding the
    uint32 bit patterns (exact while the total is < 2^32, modulo 2^32 beyond)."""
    torch = _torch()
    if src.dtype != torch.uint8:
        raise TypeError("sat_u8 needs a uint8 tensor")
    rows, cols, spitch = _matrix(src, "src")
    if out is None:
        out = torch.empty((rows, cols), dtype=torch.int32, device=src.device)
    if out.dtype != torch.int32 or out.device != src.device:
        raise ValueError("out must be an int32 tensor on src's device")
    orows, ocols, opitch = _matrix(out, "out")
    if (orows, ocols) != (rows, cols):
        raise ValueError("out must have src's shape")
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_compute_u8(src.data_ptr(), spitch, out.data_ptr(), rows, cols, opitch,
                                        _stream_ptr(stream)), "sat_compute_u8")
    return out


def sat_f64(src, out=None, *, stream=None):
    """fp64 SAT of a 2-D float32 CUDA tensor (sat_compute_f32_f64, NEXT-3): returns float64 (rows, cols)."""
    torch = _torch()
    if src.dtype != torch.float32:
        raise TypeError("sat_f64 needs a float32 tensor")
    rows, cols, spitch = _matrix(src, "src")
    if out is None:
        out = torch.empty((rows, cols), dtype=torch.float64, device=src.device)
    if out.dtype != torch.float64 or out.device != src.device:
        raise ValueError("out must be a float64 tensor on src's device")
    orows, ocols, opitch = _matrix(out, "out")
    if (orows, ocols) != (rows, cols):
        raise ValueError("out must have src's shape")
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_compute_f32_f64(src.data_ptr(), spitch, out.data_ptr(), opitch, rows, cols,
                                             _stream_ptr(stream)), "sat_compute_f32_f64")
    return out


def sat_moments(src, out=None, *, stream=None):
    """Summed-area variance shadow map moments of a 2-D float32 CUDA tensor (sat_compute_moments_f32):
    returns float32 (rows, cols, 2) with [..., 0] = SAT(a) and [..., 1] = SAT(a*a)."""
    torch = _torch()
    if src.dtype != torch.float32:
        raise TypeError("sat_moments needs a float32 tensor")
    rows, cols, spitch = _matrix(src, "src")
    if out is None:
        out = torch.empty((rows, cols, 2), dtype=torch.float32, device=src.device)
    if out.dtype != torch.float32 or out.device != src.device or out.dim() != 3 or tuple(out.shape) != (rows, cols, 2) \
            or out.stride(2) != 1 or out.stride(1) != 2 or (rows > 1 and out.stride(0) % 2):
        raise ValueError("out must be a float32 (rows, cols, 2) tensor of contiguous pairs on src's device")
    opitch = out.stride(0) // 2 if rows > 1 else cols
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_compute_moments_f32(src.data_ptr(), spitch, out.data_ptr(), opitch, rows, cols,
                                                 _stream_ptr(stream)), "sat_compute_moments_f32")
    return out


def box_sum(b, rh: int, rw: int, out=None, *, stream=None):
    """Box filter from a SAT ``b``: out[i][j] = sum of the input over the window
    [i-rh, i+rh] x [j-rw, j+rw] clipped to the matrix.  ``out`` must not be ``b``."""
    torch = _torch()
    rows, cols, pitch = _matrix(b, "b")
    if out is None:
        out = torch.empty_strided((rows, cols), (pitch, 1), dtype=b.dtype, device=b.device)
    orows, ocols, opitch = _matrix(out, "out")
    if (orows, ocols, opitch) != (rows, cols, pitch) or out.dtype != b.dtype or out.device != b.device:
        raise ValueError("out must match b in shape, row stride, dtype and device")
    with torch.cuda.device(b.device):
        check(_lib.lib().sat_box_sum(_dtype_code(b), b.data_ptr(), out.data_ptr(), rows, cols, pitch, rh, rw,
                                     _stream_ptr(stream)), "sat_box_sum")
    return out


def rect_sums(b, rects, out=None, *, stream=None):
    """Rectangle sums from a SAT ``b``: ``rects`` is an (n, 4) int64 CUDA tensor of
    (u, d, l, r), each row giving the sum over u < i <= d, l < j <= r."""
    torch = _torch()
    rows, cols, pitch = _matrix(b, "b")
    if rects.dtype != torch.int64 or rects.dim() != 2 or rects.shape[1] != 4 or not rects.is_contiguous() \
            or rects.device != b.device:
        raise ValueError("rects must be a contiguous (n, 4) int64 tensor on b's device")
    n = rects.shape[0]
    if out is None:
        out = torch.empty(n, dtype=b.dtype, device=b.device)
    _check_vec_out(out, n, b.dtype, b.device)
    with torch.cuda.device(b.device):
        check(_lib.lib().sat_rect_sums(_dtype_code(b), b.data_ptr(), rows, cols, pitch, rects.data_ptr(), n,
                                       out.data_ptr(), _stream_ptr(stream)), "sat_rect_sums")
    return out


def strip_colsum(src, out=None, *, stream=None):
    """Column sums of a strip (device), deterministic order."""
    torch = _torch()
    rows, cols, pitch = _matrix(src, "src")
    if out is None:
        out = torch.empty(cols, dtype=src.dtype, device=src.device)
    _check_vec_out(out, cols, src.dtype, src.device)
    with torch.cuda.device(src.device):
        check(_lib.lib().sat_strip_colsum(_dtype_code(src), src.data_ptr(), out.data_ptr(), rows, cols, pitch,
                                          _stream_ptr(stream)), "sat_strip_colsum")
    return out


def carry_prefix(gathered, rank: int, out=None, *, stream=None):
    """Carry row of ``rank`` from the (nranks x cols) gathered column sums (device)."""
    torch = _torch()
    if gathered.dim() != 2 or not gathered.is_contiguous() or not gathered.is_cuda:
        raise ValueError("gathered must be a contiguous (nranks, cols) CUDA tensor")
    nranks, cols = gathered.shape
    if out is None:
        out = torch.empty(cols, dtype=gathered.dtype, device=gathered.device)
    _check_vec_out(out, cols, gathered.dtype, gathered.device)
    with torch.cuda.device(gathered.device):
        check(_lib.lib().sat_carry_prefix(_dtype_code(gathered), gathered.data_ptr(), nranks, rank, cols,
                                          out.data_ptr(), _stream_ptr(stream)), "sat_carry_prefix")
    return out


def strip_bounds(rows: int, world: int, rank: int) -> tuple[int, int]:
    """Horizontal strip of ``rank`` when ``rows`` global rows are split over ``world`` ranks:
    returns (row0, nrows).  Strips are ceil(rows/world) tall; the last ones may be shorter or empty."""
    if world < 1 or not 0 <= rank < world or rows < 0:
        raise ValueError("bad strip partition arguments")
    h = -(-rows // world)
    row0 = min(rank * h, rows)
    return row0, min(h, rows - row0)


def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 of ``group`` draws a 128-byte NCCL unique id (sat_comm_get_unique_id) and the group
    broadcasts it (over the group's own backend: NCCL needs a CUDA tensor, gloo a CPU one)."""
    import torch.distributed as dist

    torch = _torch()
    buf = ctypes.create_string_buffer(128)
    if dist.get_rank(group) == 0:
        check(_lib.lib().sat_comm_get_unique_id(buf), "sat_comm_get_unique_id")
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")
    t = torch.tensor(list(buf.raw), dtype=torch.uint8, device=dev)
    dist.broadcast(t, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    return bytes(t.cpu().tolist())


def strip_layout(rows: int, cols: int, dtype_code: int, group=None) -> tuple[int, int]:
    """Collective host-side check of a strip partition: every rank passes its own strip height and the
    common column count / dtype.  Returns (row0 of this rank, total rows).  Raises ValueError on every
    rank if the ranks disagree on cols or dtype (sat_compute_sharded requires equal cols)."""
    import torch.distributed as dist

    torch = _torch()
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")
    mine = torch.tensor([rows, cols, dtype_code], dtype=torch.int64, device=dev)
    allv = [torch.empty_like(mine) for _ in range(world)]
    dist.all_gather(allv, mine, group=group)
    table = [tuple(int(x) for x in v.cpu().tolist()) for v in allv]
    if any(c != table[0][1] or d != table[0][2] for _, c, d in table):
        raise ValueError(f"strip partition mismatch across ranks: (rows, cols, dtype) = {table}")
    if any(r < 0 for r, _, _ in table):
        raise ValueError("negative strip height")
    row0 = sum(r for r, _, _ in table[:rank])
    return row0, sum(r for r, _, _ in table)


class Comm:
    """NCCL communicator for sat_sharded, bootstrapped over a torch process group: rank 0 creates the
    128-byte NCCL id, the group broadcasts it, every rank calls sat_comm_init collectively."""

    def __init__(self, group=None):
        import torch.distributed as dist

        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        raw = broadcast_unique_id(group)
        self._h = ctypes.c_void_p()
        check(_lib.lib().sat_comm_init(ctypes.byref(self._h), raw, self.world, self.rank), "sat_comm_init")

    def close(self):
        if self._h:
            _lib.lib().sat_comm_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


def sat_sharded(strip, out=None, *, comm: Comm, stream=None, check_layout: bool = False):
    """Strip-partitioned SAT: this rank's horizontal strip in, this rank's strip of the global SAT out.
    Collective over ``comm`` (call on every rank in the same order, equal column counts).  With
    ``check_layout`` the ranks first verify the partition (strip_layout, one small collective)."""
    torch = _torch()
    rows, cols, pitch = _matrix(strip, "strip") if strip.shape[0] > 0 else (0, strip.shape[1], strip.shape[1])
    if check_layout:
        strip_layout(rows, cols, _dtype_code(strip), comm.group)
    if out is None:
        out = torch.empty_strided((rows, cols), (pitch, 1), dtype=strip.dtype, device=strip.device)
    if out.dtype != strip.dtype or out.device != strip.device or tuple(out.shape) != (rows, cols) or \
            (rows > 0 and _matrix(out, "out")[2] != pitch):
        raise ValueError("out must match strip in shape, row stride, dtype and device")
    with torch.cuda.device(strip.device):
        check(_lib.lib().sat_compute_sharded(comm._h, _dtype_code(strip), strip.data_ptr(), out.data_ptr(), rows,
                                             cols, pitch, _stream_ptr(stream)), "sat_compute_sharded")
    return out


def exchange_blobs(blob: bytes, group=None) -> list[bytes]:
    """All-gather one fixed-size byte string per rank over a torch process group (host-side plumbing of
    the chained partition: the 64-byte CUDA IPC handles).  Works over nccl (CUDA tensors) and gloo."""
    import torch.distributed as dist

    torch = _torch()
    world = dist.get_world_size(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")
    mine = torch.tensor(list(blob), dtype=torch.uint8, device=dev)
    allv = [torch.empty_like(mine) for _ in range(world)]
    dist.all_gather(allv, mine, group=group)
    return [bytes(v.cpu().tolist()) for v in allv]


class Chain:
    """Chained strip partition (sat_chain_*, NEXT-1): rank r's strip of a horizontally partitioned
    matrix, computed in one pass with the strip column sums of the ranks above arriving through
    peer-mapped memory inside the kernels.  ``Chain(cols, group=g)`` is collective over a torch process
    group (one process per GPU; the IPC handles are all-gathered over ``g``); ``Chain.local(n, cols)``
    builds the n ranks of an emulated chain inside ONE process on the current device."""

    def __init__(self, cols: int, group=None, *, _local=None):
        if _local is not None:
            self.nranks, self.rank = _local
            self.group = None
        else:
            import torch.distributed as dist

            self.group = group
            self.nranks, self.rank = dist.get_world_size(group), dist.get_rank(group)
        self.cols = cols
        self._h = ctypes.c_void_p()
        check(_lib.lib().sat_chain_create(self.nranks, self.rank, cols, ctypes.byref(self._h)), "sat_chain_create")
        if _local is None:
            handle = ctypes.create_string_buffer(64)
            check(_lib.lib().sat_chain_export(self._h, handle), "sat_chain_export")
            blobs = exchange_blobs(handle.raw, group)
            check(_lib.lib().sat_chain_connect(self._h, b"".join(blobs)), "sat_chain_connect")

    @classmethod
    def local(cls, n: int, cols: int) -> list["Chain"]:
        chains = [cls(cols, _local=(n, r)) for r in range(n)]
        arr = (ctypes.c_void_p * n)(*[c._h.value for c in chains])
        check(_lib.lib().sat_chain_connect_local(arr, n), "sat_chain_connect_local")
        return chains

    def close(self):
        if self._h:
            _lib.lib().sat_chain_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


def sat_chained(strip, out=None, *, chain: Chain, stream=None):
    """This rank's strip of the SAT of the row-stacked strips of all ranks (sat_compute_chained).  Collective
    over the chain (every rank, same order, >= 1 row each)."""
    torch = _torch()
    rows, cols, pitch = _matrix(strip, "strip")
    if out is None:
        out = torch.empty_strided((rows, cols), (pitch, 1), dtype=strip.dtype, device=strip.device)
    orows, ocols, opitch = _matrix(out, "out")
    if (orows, ocols, opitch) != (rows, cols, pitch) or out.dtype != strip.dtype or out.device != strip.device:
        raise ValueError("out must match strip in shape, row stride, dtype and device")
    with torch.cuda.device(strip.device):
        check(_lib.lib().sat_compute_chained(chain._h, _dtype_code(strip), strip.data_ptr(), out.data_ptr(), rows, cols,
                                             pitch, _stream_ptr(stream)), "sat_compute_chained")
    return out


def query_plan(dtype: int, rows: int, cols: int, pitch: int | None = None, src_ptr: int = 0,
               dst_ptr: int = 0) -> dict:
    """What sat_compute would launch (tile shape, TMA or not, CTAs, tiles, aux bytes)."""
    p = SatPlan()
    check(_lib.lib().sat_query_plan(dtype, rows, cols, cols if pitch is None else pitch, src_ptr or None,
                                    dst_ptr or None, ctypes.byref(p)), "sat_query_plan")
    return {f: getattr(p, f) for f, _ in SatPlan._fields_}


def set_tuning(variant: int = -1, order: int = 0, ctas_per_sm: int = 0) -> None:
    check(_lib.lib().sat_set_tuning(variant, order, ctas_per_sm), "sat_set_tuning")


def set_max_ctas(max_ctas: int = 0) -> None:
    """Cap the persistent grid (0 = no cap); 1 = single-CTA forward-progress test."""
    check(_lib.lib().sat_set_max_ctas(max_ctas), "sat_set_max_ctas")


def num_variants() -> int:
    return _lib.lib().sat_num_variants()


def variant_info(v: int) -> tuple[int, int]:
    tr, tc = ctypes.c_int32(), ctypes.c_int32()
    check(_lib.lib().sat_variant_info(v, ctypes.byref(tr), ctypes.byref(tc)), "sat_variant_info")
    return tr.value, tc.value


def debug_tile_order(R: int, C: int, order: int = 0, device=None):
    """The kernel's serial -> (I, J) map evaluated on the GPU: int32 tensor (R*C, 2)."""
    torch = _torch()
    out = torch.empty((R * C, 2), dtype=torch.int32, device=device or "cuda")
    with torch.cuda.device(out.device):
        check(_lib.lib().sat_debug_tile_order(R, C, order, out.data_ptr(), _stream_ptr(None)), "sat_debug_tile_order")
    return out


def debug_occupy(ctas: int, ns: int, smem_bytes: int = 200 * 1024, *, stream=None) -> None:
    """Test hook (sat_debug_occupy): ``ctas`` CTAs holding ``smem_bytes`` of shared memory each spin for
    ``ns`` nanoseconds on ``stream`` (adversarial SM occupancy for the forward-progress tests)."""
    check(_lib.lib().sat_debug_occupy(ctas, ns, smem_bytes, _stream_ptr(stream)), "sat_debug_occupy")


def debug_workspace(stream=None, words: bool = True):
    """Test hook (sat_debug_workspace): the published aggregate words of the last sat_compute launch on
    ``stream`` (current stream by default).  Returns (info dict, numpy uint64 array or None): row slots
    [R*C][tile_rows], column slots [R*C][tile_cols], corner slots [R*C]."""
    import numpy as np

    info = _lib.SatWsInfo()
    sp = _stream_ptr(stream)
    check(_lib.lib().sat_debug_workspace(sp, None, 0, ctypes.byref(info)), "sat_debug_workspace")
    d = {f: getattr(info, f) for f, _ in _lib.SatWsInfo._fields_}
    if not words:
        return d, None
    buf = np.empty(max(1, d["words"]), dtype=np.uint64)
    check(_lib.lib().sat_debug_workspace(sp, buf.ctypes.data, buf.size, ctypes.byref(info)), "sat_debug_workspace")
    return d, buf[: d["words"]]


def release_stream_workspace(stream=None) -> None:
    check(_lib.lib().sat_release_stream_workspace(_stream_ptr(stream)), "sat_release_stream_workspace")


def release_workspaces() -> None:
    check(_lib.lib().sat_release_workspaces(), "sat_release_workspaces")


def version() -> int:
    return _lib.lib().sat_version()
