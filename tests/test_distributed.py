"""Multi-process host logic of the strip-partitioned path (BASELINE.json configs[4]) on CPU with the
gloo backend, world size 2 and 3: the NCCL id bootstrap, the strip partition check, and the carry
exchange protocol (which ranks' column sums enter a rank's carry, in which order) replayed with the
oracle's arithmetic through real torch.distributed collectives.  On a GPU box,
test_gather_path_multiprocess_libsat_kernels runs the same exchange with libsat's own device kernels in
2 / 3 processes (gloo in place of ncclAllGather); the chained path's two-process CUDA IPC test is in
tests/test_gpu_chain.py."""
import os
import socket
import traceback

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(world, fn, *args):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_entry, args=(r, world, port, fn, args, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    errs = [r for r in results if r[1] is not None]
    assert not errs, errs[0][1]
    return {r[0]: r[2] for r in results}


def _entry(rank, world, port, fn, args, q):
    try:
        import sys
        from pathlib import Path

        root = str(Path(__file__).resolve().parent.parent)
        sys.path.insert(0, root)
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        out = fn(rank, world, *args)
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, None, out))
    except Exception:
        q.put((rank, traceback.format_exc(), None))


# ----------------------------------------------------------------------------------------- workers
def _w_unique_id(rank, world):
    import paper_conf_ipps_emotofthni18_b200 as sat

    raw = sat.broadcast_unique_id()
    assert len(raw) == 128
    gathered = [None] * world
    dist.all_gather_object(gathered, raw)
    assert all(g == gathered[0] for g in gathered)
    return raw.hex()


def _w_layout(rank, world, heights, cols_per_rank):
    import paper_conf_ipps_emotofthni18_b200 as sat

    try:
        row0, total = sat.strip_layout(heights[rank], cols_per_rank[rank], sat.SAT_INT32)
        return ("ok", row0, total)
    except ValueError as e:
        return ("mismatch", str(e))


def _w_carry_exchange(rank, world, rows, cols, seed):
    """The exchange of sat_compute_sharded with oracle arithmetic: colsum of my strip -> all_gather ->
    C_r = sum_{g<r} colsum_g (ascending g) -> carry = row-wise prefix of C_r; then my strip of the SAT
    is carry + SAT(strip).  Checked against the oracle SAT of the whole matrix."""
    import oracle
    import paper_conf_ipps_emotofthni18_b200 as sat
    import satgen

    row0, n = sat.strip_bounds(rows, world, rank)
    strip = satgen.gen_host(n, cols, seed, "u32", row0=row0)
    r0_chk, total = sat.strip_layout(n, cols, sat.SAT_INT32)
    assert (r0_chk, total) == (row0, rows)
    colsum = oracle.strip_carry_u32(strip, cols)  # column sums of my strip (mod 2^32)
    gathered = [torch.zeros(cols, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(gathered, torch.from_numpy(colsum.astype(np.int64)))
    C = np.zeros(cols, dtype=np.uint64)
    for g in range(rank):  # ascending rank order (reading R12)
        C = (C + gathered[g].numpy().astype(np.uint64)) % (1 << 32)
    carry = oracle.row_prefix_u32(C.astype(np.uint32)[None, :])[0]
    mine = (oracle.sat_u32(strip).astype(np.uint64) + carry.astype(np.uint64)[None, :]) % (1 << 32)
    full = oracle.sat_u32(satgen.gen_host(rows, cols, seed, "u32"))
    assert (mine.astype(np.uint32) == full[row0:row0 + n]).all()
    return int(mine.astype(np.uint64).sum() % (1 << 32)) if n else 0


# ----------------------------------------------------------------------------------------- tests
def test_unique_id_broadcast_gloo():
    ids = _run(2, _w_unique_id)
    assert ids[0] == ids[1]


def test_strip_layout_consistent_and_mismatch():
    res = _run(3, _w_layout, [5, 7, 0], [11, 11, 11])
    assert res[0] == ("ok", 0, 12) and res[1] == ("ok", 5, 12) and res[2] == ("ok", 12, 12)
    bad = _run(2, _w_layout, [4, 4], [11, 12])
    assert all(r[0] == "mismatch" for r in bad.values())


@pytest.mark.parametrize("world", [2, 3])
def test_carry_exchange_protocol_gloo(world):
    _run(world, _w_carry_exchange, 61, 45, 1447 + world)


# ----------------------------------------------------------------------------- chained partition: handle exchange
def _blob_worker(rank, port, q):
    try:
        import os
        import sys
        from pathlib import Path

        sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
        import torch.distributed as dist

        import paper_conf_ipps_emotofthni18_b200 as sat

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=2)
        blob = bytes((rank * 37 + i) % 256 for i in range(64))  # stands in for a 64-byte CUDA IPC handle
        got = sat.exchange_blobs(blob, None)
        dist.destroy_process_group()
        q.put((rank, got))
    except Exception:
        import traceback

        q.put((rank, traceback.format_exc()))


def test_chain_handle_exchange_gloo_world2():
    """The host plumbing of Chain(group): every rank receives every rank's 64-byte handle, in rank order."""
    import socket

    import torch.multiprocessing as mp

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_blob_worker, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=30)
    want = [bytes((r * 37 + i) % 256 for i in range(64)) for r in range(2)]
    assert out[0] == want and out[1] == want


# ----------------------------------------------------------------------------- gather path through libsat's kernels
def _w_gather_path_libsat(rank, world, rows, cols, seed, dist_name):
    """The exchange of sat_compute_sharded with libsat's OWN device kernels in every process -- strip column
    sums (sat_strip_colsum), carry row (sat_carry_prefix), single pass with the carry (sat_compute) --
    and gloo standing in for ncclAllGather (this pool gives one GPU per call; NCCL refuses two ranks on one
    device).  Each rank checks its strip against the oracle SAT of the whole matrix."""
    import oracle
    import paper_conf_ipps_emotofthni18_b200 as sat
    import satgen

    torch.cuda.set_device(0)
    row0, n = sat.strip_bounds(rows, world, rank)
    strip = satgen.gen_host(n, cols, seed, dist_name, row0=row0)
    x = torch.from_numpy(strip).cuda()
    colsum = sat.strip_colsum(x)
    gathered = [torch.zeros(cols, dtype=x.dtype) for _ in range(world)]
    dist.all_gather(gathered, colsum.cpu())
    carry = sat.carry_prefix(torch.stack(gathered).cuda(), rank)
    got = sat.sat(x, carry=carry).cpu().numpy()
    full = satgen.gen_host(rows, cols, seed, dist_name)
    if dist_name == "u32":
        assert (got == oracle.sat_i32(full)[row0:row0 + n]).all()
    else:
        b, ab = oracle.sat_f32(full)
        tol = oracle.f32_tolerance(ab, rows, cols)[row0:row0 + n]
        assert (np.abs(got.astype(np.float64) - b[row0:row0 + n]) <= tol).all()
    return n


@pytest.mark.gpu
@pytest.mark.parametrize("world,dist_name", [(2, "u32"), (3, "u32"), (2, "fsym")])
def test_gather_path_multiprocess_libsat_kernels(world, dist_name):
    res = _run(world, _w_gather_path_libsat, 2500, 3100, 4141 + world, dist_name)
    assert sum(res.values()) == 2500
