"""Chained strip partition (sat_compute_chained) against the oracle.

The N ranks of a chain are emulated on the one GPU of this box: ``Chain.local`` connects N chains of one
process through their device buffers (the kernels' "peer" stores then land in the same HBM), which runs
exactly the in-kernel protocol of the multi-GPU path -- column-major tiles, strip-local look-backs,
bottom tiles pushing epoch-tagged column sums into downstream inboxes, inbox polling, back-pressure.
Ranks run one after the other on one stream, concurrently on N streams (grid split N ways, so the
ranks' kernels are co-resident), with one CTA per rank, and over several calls without host syncs (the
double-buffered inbox and its back-pressure).  A two-process test exercises the CUDA IPC path.
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


def _strips(sat, a, n):
    rows = a.shape[0]
    return [sat.strip_bounds(rows, n, r) for r in range(n)]


def _check(got, a, dist):
    if dist == "u32":
        want = oracle.sat_i32(a)
        if not (got == want).all():
            bad = np.argwhere(got != want)
            raise AssertionError(f"{len(bad)} mismatches; first at {bad[0].tolist()}")
    else:
        b, ab = oracle.sat_f32(a)
        tol = oracle.f32_tolerance(ab, *a.shape)
        err = np.abs(got.astype(np.float64) - b)
        assert (err <= tol).all(), f"fp32 outside tolerance at {np.unravel_index(np.argmax(err - tol), err.shape)}"


@pytest.mark.parametrize("n,shape,dist", [(1, (300, 517), "u32"), (2, (1203, 1777), "u32"), (3, (1000, 3000), "u32"),
                                          (8, (2049, 1500), "u32"), (4, (900, 2100), "fsym"), (8, (1030, 640), "fu2")])
def test_chain_sequential_ranks(sat, n, shape, dist):
    a = satgen.gen_host(*shape, seed=600 + n, dist=dist)
    chains = sat.Chain.local(n, shape[1])
    try:
        parts = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + h])).cuda() for r0, h in _strips(sat, a, n)]
        for call in range(3):  # several calls: alternating inbox halves, epochs, back-pressure words
            outs = [sat.sat_chained(x, chain=c) for x, c in zip(parts, chains)]
            got = torch.cat(outs).cpu().numpy()
            _check(got, a, dist)
    finally:
        for c in chains:
            c.close()


@pytest.mark.parametrize("n,ctas", [(2, 0), (4, 0), (8, 0), (3, 1), (8, 1)])
def test_chain_concurrent_ranks(sat, n, ctas):
    """All ranks' kernels in flight at once on their own streams, each with 148/n (or 1) CTAs, three calls
    queued back to back without host synchronisation."""
    rows, cols = 4100, 2600
    a = satgen.gen_host(rows, cols, seed=700 + n, dist="u32")
    chains = sat.Chain.local(n, cols)
    streams = [torch.cuda.Stream() for _ in range(n)]
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    sat.set_max_ctas(ctas if ctas else max(1, sms // n))
    try:
        parts = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + h])).cuda() for r0, h in _strips(sat, a, n)]
        torch.cuda.synchronize()
        outs = [[None] * n for _ in range(3)]
        for call in range(3):
            for r in range(n):
                with torch.cuda.stream(streams[r]):
                    outs[call][r] = sat.sat_chained(parts[r], chain=chains[r], stream=streams[r])
        torch.cuda.synchronize()
        want = oracle.sat_i32(a)
        for call in range(3):
            got = torch.cat(outs[call]).cpu().numpy()
            assert (got == want).all(), f"call {call}"
    finally:
        sat.set_max_ctas(0)
        for c in chains:
            c.close()


def test_chain_strip_of_64k_columns(sat):
    """configs[4]'s 64K-column width: 2 ranks x 1024 rows x 65536 int32, every element."""
    rows, cols, n = 2048, 65536, 2
    a = satgen.gen_host(rows, cols, seed=800, dist="u32")
    chains = sat.Chain.local(n, cols)
    try:
        parts = [torch.from_numpy(np.ascontiguousarray(a[r0:r0 + h])).cuda() for r0, h in _strips(sat, a, n)]
        got = torch.cat([sat.sat_chained(x, chain=c) for x, c in zip(parts, chains)]).cpu().numpy()
        _check(got, a, "u32")
    finally:
        for c in chains:
            c.close()


def test_chain_argument_errors(sat):
    chains = sat.Chain.local(2, 500)
    try:
        x = torch.zeros((10, 400), dtype=torch.int32, device="cuda")
        with pytest.raises(sat.SatError):
            sat.sat_chained(x, chain=chains[0])  # cols differ from the chain's
        lone = sat.Chain(500, _local=(2, 1))  # never connected
        with pytest.raises(sat.SatError):
            sat.sat_chained(torch.zeros((10, 500), dtype=torch.int32, device="cuda"), chain=lone)
        lone.close()
    finally:
        for c in chains:
            c.close()


# ----------------------------------------------------------------------------- two processes, CUDA IPC
def _ipc_rank(rank, port, q):
    try:
        import os
        import sys
        from pathlib import Path

        sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
        import torch
        import torch.distributed as dist

        import paper_conf_ipps_emotofthni18_b200 as sat
        import satgen

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=2)
        rows, cols = 700, 1300
        r0, h = sat.strip_bounds(rows, 2, rank)
        x = torch.from_numpy(satgen.gen_host(h, cols, seed=900, dist="u32", row0=r0)).cuda()
        sat.set_max_ctas(16)  # both processes' kernels fit on the GPU at once
        chain = sat.Chain(cols)
        outs = []
        for _ in range(2):
            outs.append(sat.sat_chained(x, chain=chain))
        torch.cuda.synchronize()
        dist.barrier()
        chain.close()
        dist.destroy_process_group()
        q.put((rank, "ok", [o.cpu().numpy() for o in outs]))
    except Exception:
        import traceback

        q.put((rank, "error", traceback.format_exc()))


def test_chain_two_processes_ipc():
    """Two processes on this GPU, handles all-gathered over gloo, peers opened with cudaIpcOpenMemHandle."""
    import socket

    import torch.multiprocessing as mp

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_rank, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(2):
            rank, status, payload = q.get(timeout=240)
            assert status == "ok", payload
            res[rank] = payload
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    a = satgen.gen_host(700, 1300, seed=900, dist="u32")
    want = oracle.sat_i32(a)
    for call in range(2):
        got = np.concatenate([res[0][call], res[1][call]])
        assert (got == want).all(), f"call {call}"
