#!/usr/bin/env python
"""bench.py -- single-pass SAT throughput on B200 (driver contract: one JSON line from rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--dtype f32|i32] [--size S] [--impl ours|reference]
    python bench.py --sweep            # extra: the paper's size sweep 256^2..32K^2, one JSON line per size

Step = one pass of the whole hot path over one matrix (tile counter, TMA
loads, local SAT, look-backs, corrections, TMA stores -- one kernel launch) on synthetic inputs
generated in HBM by the seeded generator.  N = 1: the 32K x 32K matrix the BASELINE.json metric is
quoted on.  N > 1 (torchrun, one process per GPU): the 64K x 64K strip-partitioned configuration
(BASELINE.json configs[4]); each rank owns a horizontal strip, one step = sat_compute_sharded
(strip column sums -> NCCL allgather -> carry row -> single pass with the carry).

value = elements of the whole job / (max over ranks of the device time per step), Gelem/s.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

METRIC = "SAT Gelem/s and HBM GB/s at 32K×32K vs D2D memcpy; 1/2/4/8 B200 scaling"
UNIT = "Gelem/s"
BYTES_PER_ELEM = 8  # algorithmic: 4 B read + 4 B written per element (P:5)
PAPER_32K_F32_GELEMS = 32768 * 32768 / 15.8e-3 / 1e9  # Table III: 15.8 ms on TITAN V (context)


def measured_peaks() -> tuple[float, str]:
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms while the timed region runs."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines: list[str] = []
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict | None:
        if not self.proc:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for name, val in zip(names, parts[4:8]):
                if val.lower().startswith("active"):
                    reasons.add(name)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------- CPU baseline (oracle)
def host_cpu() -> dict:
    model = "unknown"
    try:
        for ln in Path("/proc/cpuinfo").read_text().splitlines():
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


class pinned_to_one_core:
    """Run the single-threaded oracle pinned to one host core (sched_setaffinity), then restore."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        self.core = min(self.prev)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.prev)


def cpu_oracle_sample(rows: int, cols: int, dtype: str, target_s: float = 12.0) -> dict:
    """Time the CPU oracle (oracle/, as it stands, single thread pinned to one core) on a bounded sample
    of the workload: the first `h` rows (all columns) of the same seeded matrix, h chosen for ~target_s of
    CPU work."""
    import oracle
    import satgen

    dist = "f01" if dtype == "f32" else "u32"

    def run(h):
        a = satgen.gen_host(h, cols, 1447, dist)
        t0 = time.perf_counter()
        if dtype == "f32":
            oracle.sat_f32(a, with_abs=False)
        else:
            oracle.sat_u32(a)
        return time.perf_counter() - t0

    with pinned_to_one_core() as pin:
        h = min(rows, 64)
        t = run(h)
        while t < 0.5 and h < rows:
            h = min(rows, h * 4)
            t = run(h)
        rate = h * cols / t
        h2 = int(min(rows, max(h, rate * target_s / cols)))
        if h2 > h:
            h, t = h2, run(h2)
        core = pin.core
    return {"value": h * cols / t / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"first {h} of {rows} rows x {cols} cols ({dtype}, seed 1447), in-memory C oracle "
                      f"(column-then-row, single thread pinned to core {core}), {t:.2f} s",
            **host_cpu()}


# ------------------------------------------------------------------------------------- helpers
def order_name(order: int) -> str:
    """Tile order of the plan: 0 anti-diagonal (Fig. 9), 1 row-major, (g << 8) diagonal of g-tile groups."""
    g = (order >> 8) & 255
    if (order & 15) == 0 and g > 1:
        return f"anti-diagonal of {g}-tile groups"
    return ["anti-diagonal", "row-major"][order & 15]


def load_ncu_traffic(workload: str):
    """DRAM read + write bytes per launch of this workload's SAT kernel from the committed ncu capture
    (profiles/ncu_summary.json, one `ncu --set full` launch of the same kernel and configuration)."""
    p = ROOT / "profiles" / "ncu_summary.json"
    if not p.exists():
        return None, None
    try:
        d = json.loads(p.read_text())
        e = d.get(workload)
        if e is None:
            return None, None
        return e.get("dram_bytes_per_launch"), f"profiles/ncu_summary.json ({e.get('source', 'ncu --set full')})"
    except Exception:
        return None, None


def dist_info():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ------------------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank, world, _ = dist_info()
    if rank != 0:
        return 0
    import numpy as np  # noqa: F401

    import oracle
    import satgen

    n = args.size or 32768
    rows = cols = n
    dtype = args.dtype
    dist = "f01" if dtype == "f32" else "u32"
    # each step: the oracle on a bounded sample (the first h rows) of the same workload
    h = max(1, min(rows, int(os.environ.get("SAT_REF_ROWS", "2048"))))
    a = satgen.gen_host(h, cols, 1447, dist)
    f = (lambda: oracle.sat_f32(a, with_abs=False)) if dtype == "f32" else (lambda: oracle.sat_u32(a))
    times = []
    with pinned_to_one_core():
        for _ in range(args.warmup):
            f()
        for _ in range(args.steps):
            t0 = time.perf_counter()
            f()
            times.append(time.perf_counter() - t0)
    ms = statistics.mean(times) * 1e3
    value = h * cols / (ms / 1e3) / 1e9
    sample = (f"first {h} of {rows} rows x {cols} cols per step ({dtype}, seed 1447), single-thread C oracle "
              f"pinned to one core")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak" if world == 1 else "strong",
        "vs_baseline": None, "dtype": "f64" if dtype == "f32" else "u32", "data": "synthetic",
        "config": {"workload": f"{n}x{n} {dtype} SAT (sampled rows)", "rows": rows, "cols": cols},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample, **host_cpu()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--dtype", choices=["f32", "i32"], default="f32")
    ap.add_argument("--size", type=int, default=0, help="matrix side (default 32768; 65536 when N>1)")
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--sweep", action="store_true")
    ap.add_argument("--no-extras", action="store_true", help="skip the other BASELINE configs (4K^2, sweep, 64K^2)")
    ap.add_argument("--sharded", choices=["chain", "gather"], default="chain",
                    help="N>1: chained strips in one pass (default) or column sums + NCCL all-gather + SAT")
    ap.add_argument("--variant", type=int, default=-1)
    ap.add_argument("--order", type=int, default=0)
    ap.add_argument("--ctas-per-sm", type=int, default=0)
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)

    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_emotofthni18_b200 as sat
    import satgen

    rank, world, local = dist_info()
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    sat.set_tuning(args.variant, args.order, args.ctas_per_sm)

    if args.sweep:
        return run_sweep(args, sat, satgen, torch)

    n = args.size or (32768 if world == 1 else 65536)
    rows = cols = n
    tdt = torch.float32 if args.dtype == "f32" else torch.int32
    dist_name = "f01" if args.dtype == "f32" else "u32"
    stream = torch.cuda.current_stream()

    if world == 1:
        row0, nrows = 0, rows
    else:
        row0, nrows = sat.strip_bounds(rows, world, rank)
    x = torch.empty((nrows, cols), dtype=torch.int32, device=dev)
    satgen.fill_tensor(x, 1447, dist_name, row0=row0)
    x = x.view(tdt)
    y = torch.empty_like(x)
    comm = chain = None
    fallback = None
    if world > 1 and args.sharded == "chain":
        try:
            chain = sat.Chain(cols)
        except sat.SatError as e:  # e.g. CUDA IPC between the ranks' GPUs refused: every rank falls back
            fallback = f"chained strips unavailable ({e}); NCCL gather path"
        ok = torch.tensor([0 if fallback else 1], dtype=torch.int32, device=dev)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if int(ok.item()) == 0:
            if chain is not None:
                chain.close()
                chain = None
            fallback = fallback or "chained strips unavailable on another rank; NCCL gather path"
    if world > 1 and chain is None:
        comm = sat.Comm()

    def step():
        if comm is not None:
            sat.sat_sharded(x, out=y, comm=comm)
        elif chain is not None:
            sat.sat_chained(x, out=y, chain=chain)
        else:
            sat.sat(x, out=y)

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local])

    # ---- warm-up, then the timed region (K steps, barrier + sync on both sides, CUDA events)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local) if rank == 0 else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    clk = clocks.stop() if clocks else None
    ms_local = ev0.elapsed_time(ev1) / args.steps
    ms_t = torch.tensor([ms_local], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    total_elems = rows * cols
    value = total_elems / (ms / 1e3) / 1e9

    # ---- same-run D2D memcpy of this rank's matrix (the paper's yardstick)
    for _ in range(3):
        y.copy_(x)
    torch.cuda.synchronize()
    m0, m1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    m0.record(stream)
    for _ in range(args.steps):
        y.copy_(x)
    m1.record(stream)
    torch.cuda.synchronize()
    memcpy_ms = m0.elapsed_time(m1) / args.steps
    step()
    torch.cuda.synchronize()

    # ---- end to end through the C ABI with host buffers (rank 0 of N=1 only; PCIe-bound)
    e2e = None
    if rank == 0 and world == 1 and not args.no_e2e:
        try:
            e2e = run_e2e(args, sat, torch, x, rows, cols, tdt)
        except Exception as e:  # noqa: BLE001 -- report, keep the device-timed line
            e2e = {"error": f"{type(e).__name__}: {e}"[:300]}

    if rank == 0:
        peak, peak_src = measured_peaks()
        kernel_ms = ms  # one SAT launch per step (N=1)
        achieved = (nrows * cols * BYTES_PER_ELEM) / (kernel_ms / 1e3) / 1e9
        workload = f"{n}x{n} {args.dtype} SAT" + ("" if world == 1 else f" strip-partitioned over {world} GPUs")
        plan = sat.query_plan(sat.SAT_FLOAT32 if args.dtype == "f32" else sat.SAT_INT32, nrows, cols, cols,
                              x.data_ptr(), y.data_ptr())
        traffic, traffic_src = load_ncu_traffic(workload)
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak" if world == 1 else "strong",
            "vs_baseline": (value / PAPER_32K_F32_GELEMS) if (world == 1 and n == 32768 and args.dtype == "f32") else None,
            "dtype": "f32" if args.dtype == "f32" else "u32",
            "data": "synthetic (seeded splitmix64 counter generator, uniform; generated in HBM)",
            "config": {"workload": workload, "rows": rows, "cols": cols, "pitch": cols,
                       "tile": [plan["tile_rows"], plan["tile_cols"]], "ctas": plan["ctas"],
                       "variant": plan["variant"], "order": order_name(plan["order"]),
                       "l2": "inputs (4 B x n^2) larger than the 126 MB L2; no flush",
                       "parallelism": "single GPU" if world == 1 else
                       f"strips x{world} ({'sat_compute_chained' if chain is not None else 'sat_compute_sharded'})",
                       **({"fallback": fallback} if fallback else {})},
            "hbm_gbs": achieved,
            "memcpy": {"ms": memcpy_ms, "gbs": nrows * cols * BYTES_PER_ELEM / (memcpy_ms / 1e3) / 1e9,
                       "overhead_pct": (ms - memcpy_ms) / memcpy_ms * 100.0, "ratio": ms / memcpy_ms,
                       "gate": "<= 1.10 x memcpy (BASELINE north_star)"},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                         "peak_source": peak_src,
                         "kernel": {2: "sat_tm_kernel"}.get(plan["family"], "sat_tiles_kernel"),
                         "bytes_per_elem": BYTES_PER_ELEM,
                         "timing": "CUDA events on the launching stream around the K timed launches"},
            "gpu_launches": args.steps * (4 if comm is not None else 1),
            "clocks": clk,
            "e2e": e2e,
        }
        if world == 1 and not args.no_extras:
            del y
            line["extras"] = run_extras(args, sat, satgen, torch, x, peak)
        if world == 1 and not args.no_cpu:
            try:
                line["cpu_baseline"] = cpu_oracle_sample(rows, cols, args.dtype)
            except Exception as e:  # noqa: BLE001
                line["cpu_baseline"] = {"error": f"{type(e).__name__}: {e}"[:300]}
        print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if chain is not None:
        chain.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


# ------------------------------------------------------------------------------------- e2e (host buffers)
def run_e2e(args, sat, torch, x, rows, cols, tdt) -> dict:
    """The public host-buffer call (sat_compute_host): pinned input, H2D + SAT + D2H inside the timed
    region, then a sampled check of the result against the oracle (first 64 rows exactly as computed by
    the streaming oracle, and the last row after feeding the oracle every row of the input)."""
    import numpy as np

    import oracle

    h_in = torch.empty((rows, cols), dtype=tdt, pin_memory=True)
    h_out = torch.empty((rows, cols), dtype=tdt, pin_memory=True)
    h_in.copy_(x)
    # PCIe roofline: plain pinned copies of the same bytes, each direction alone
    dbuf = torch.empty_like(x)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    dbuf.copy_(h_in, non_blocking=True)
    torch.cuda.synchronize()
    h2d_s = time.perf_counter() - t0
    t0 = time.perf_counter()
    h_out.copy_(dbuf, non_blocking=True)
    torch.cuda.synchronize()
    d2h_s = time.perf_counter() - t0
    # both directions at once on two streams (the pipeline's real floor if PCIe / host memory is not duplex)
    dbuf2 = torch.empty_like(x)
    h_tmp = torch.empty((rows, cols), dtype=tdt, pin_memory=True)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    with torch.cuda.stream(s1):
        dbuf.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_tmp.copy_(dbuf2, non_blocking=True)
    torch.cuda.synchronize()
    duplex_s = time.perf_counter() - t0
    del dbuf, dbuf2, h_tmp
    nbytes = rows * cols * 4
    sat.sat_host(h_in.numpy(), h_out.numpy())  # warm-up (allocates the staging buffer)
    t0 = time.perf_counter()
    for _ in range(args.e2e_steps):
        sat.sat_host(h_in.numpy(), h_out.numpy())
    e2e_s = (time.perf_counter() - t0) / args.e2e_steps
    a = h_in.numpy()
    got = h_out.numpy()
    st = oracle.Stream(cols)
    if a.dtype == np.int32:
        head_ok = bool((got[:64] == st.rows_u32(a[:64]).view(np.int32)).all())
        st.rows_u32(a[64:rows - 1], want_out=False)
        tail_ok = bool((got[rows - 1:] == st.rows_u32(a[rows - 1:]).view(np.int32)).all())
    else:
        w, ab = st.rows_f32(a[:64])
        head_ok = bool((np.abs(got[:64] - w) <= oracle.f32_tolerance(ab, rows, cols)).all())
        st.rows_f32(a[64:rows - 1], want_out=False, want_abs=False)
        w, ab = st.rows_f32(a[rows - 1:])
        tail_ok = bool((np.abs(got[rows - 1:] - w) <= oracle.f32_tolerance(ab, rows, cols)).all())
    st.close()
    h2d_gbs, d2h_gbs = nbytes / h2d_s / 1e9, nbytes / d2h_s / 1e9
    # the copies in and out overlap with each other and with the SAT; the bound is the slower direction
    pcie_floor_s = max(nbytes / (h2d_gbs * 1e9), nbytes / (d2h_gbs * 1e9))
    return {"value": rows * cols / e2e_s / 1e9, "unit": UNIT, "h2d_bytes_per_step": nbytes,
            "d2h_bytes_per_step": nbytes, "ms_per_step": e2e_s * 1e3,
            "path": "sat_compute_host (pinned host buffers; strip-pipelined H2D | SAT | D2H)",
            "pcie": {"h2d_gbs": h2d_gbs, "d2h_gbs": d2h_gbs, "floor_ms": pcie_floor_s * 1e3,
                     "frac_of_floor": pcie_floor_s / e2e_s, "duplex_ms": duplex_s * 1e3,
                     "frac_of_duplex": duplex_s / e2e_s,
                     "how": "one pinned torch copy of the same bytes per direction, wall clock; duplex = both "
                            "directions at once on two streams"},
            "check": {"first_64_rows": head_ok, "last_row": tail_ok,
                      "how": "streaming oracle over every input row; int32 bit-exact, fp32 R10 tolerance"}}


# ------------------------------------------------------------------------------------- extras
def graph_time(torch, fn, per_graph=20, reps=5) -> float:
    """Device ms per call: `per_graph` calls captured in one CUDA graph (no host launch cost), best of
    `reps` replays timed with CUDA events on the replay stream."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(per_graph):
            fn()
    g.replay()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / per_graph)
    del g
    return best


def event_time(torch, fn, reps) -> float:
    """Device ms per call: `reps` back-to-back launches between two CUDA events (after 3 warm-ups)."""
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def size_point(torch, sat, satgen, n, dtype, peak, rows=None) -> dict:
    rows = rows or n
    x = torch.empty((rows, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, 1447, "f01" if dtype == "f32" else "u32")
    if dtype == "f32":
        x = x.view(torch.float32)
    y = torch.empty_like(x)
    if rows * n <= (1 << 26):  # latency-bound sizes: device time through CUDA graphs
        t_sat = graph_time(torch, lambda: sat.sat(x, out=y))
        t_cp = graph_time(torch, lambda: y.copy_(x))
        how = "CUDA graph of 20 calls, best of 5 replays"
    else:
        reps = max(10, min(200, int(4e10 / (rows * n * 8))))
        t_sat = event_time(torch, lambda: sat.sat(x, out=y), reps)
        t_cp = event_time(torch, lambda: y.copy_(x), reps)
        how = f"{reps} back-to-back launches between CUDA events"
    gbs = rows * n * BYTES_PER_ELEM / (t_sat / 1e3) / 1e9
    plan = sat.query_plan(sat.SAT_FLOAT32 if dtype == "f32" else sat.SAT_INT32, rows, n)
    del x, y
    return {"rows": rows, "cols": n, "dtype": dtype, "sat_ms": t_sat, "memcpy_ms": t_cp,
            "overhead_pct": (t_sat - t_cp) / t_cp * 100.0, "gelems": rows * n / (t_sat / 1e3) / 1e9,
            "gbs": gbs, "frac": gbs / peak, "tile": [plan["tile_rows"], plan["tile_cols"]], "timing": how}


def run_extras(args, sat, satgen, torch, x, peak) -> dict:
    """Every other BASELINE.json config on this GPU in the same run (device time, same-run memcpy):
    configs[1] 4K^2 int32/fp32, configs[2] the paper's size sweep 256^2..32K^2 int32 (Table III analogue,
    overhead over duplication per size), int32 32K^2, and configs[4]'s 64K^2 int32 as
    a single pass on one GPU (the 'linear' baseline of the strip-partitioned scaling)."""
    del x
    torch.cuda.empty_cache()
    out = {}

    def guard(name, fn):  # one failing extra (e.g. memory on a smaller GPU) must not cost the whole line
        try:
            out[name] = fn()
        except Exception as e:  # noqa: BLE001
            out[name] = {"error": f"{type(e).__name__}: {e}"[:300]}
            torch.cuda.synchronize()
            torch.cuda.empty_cache()

    guard("c1_4k", lambda: {d: size_point(torch, sat, satgen, 4096, d, peak) for d in ("i32", "f32")})
    guard("i32_32k", lambda: size_point(torch, sat, satgen, 32768, "i32", peak))
    guard("sweep_i32", lambda: [size_point(torch, sat, satgen, 1 << k, "i32", peak) for k in range(8, 16)])
    single = {}

    def single_64k():
        # 64K^2 int32 single GPU, in place (16 GiB) against a 16 GiB copy
        n = 65536
        xx = torch.empty((n, n), dtype=torch.int32, device="cuda")
        satgen.fill_tensor(xx, 1447, "u32")
        t_sat = event_time(torch, lambda: sat.sat(xx, out=xx), 5)
        yy = torch.empty_like(xx)
        t_cp = event_time(torch, lambda: yy.copy_(xx), 5)
        del xx, yy
        torch.cuda.empty_cache()
        single["ms"] = t_sat
        gbs = n * n * BYTES_PER_ELEM / (t_sat / 1e3) / 1e9
        return {"rows": n, "cols": n, "sat_ms": t_sat, "memcpy_ms": t_cp,
                "overhead_pct": (t_sat - t_cp) / t_cp * 100.0, "gbs": gbs, "frac": gbs / peak,
                "note": "in place; 5 launches between CUDA events"}

    guard("i32_64k_single_gpu", single_64k)
    if "ms" in single:
        guard("chain_64k", lambda: chain_projection(torch, sat, satgen, 65536, single["ms"]))
    guard("next_paths_32k", lambda: next_paths(torch, sat, satgen, 32768, peak))
    return out


def next_paths(torch, sat, satgen, n, peak) -> dict:
    """SURVEY Sec. 8(f) rows beyond the hot path, device time at n x n (median of 10 after 3 warm-ups),
    algorithmic GB/s against the measured copy peak and a same-bytes torch copy: u8 -> uint32 integral
    image (NEXT-3, 1 + 4 B/elem; yardstick the u8 -> int32 widening copy), fp32 -> fp64 SAT and SAVSM
    moments (NEXT-3, 4 + 8 B/elem; yardstick the fp32 -> fp64 widening copy), box filter r = 8 / 64
    (NEXT-4, 4 + 4 B/elem), batched 256^2 int32 and u8 (NEXT-2)."""
    import statistics

    def med(fn, reps=10):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)

    def entry(ms, bpe, yard_ms, yard):
        gbs = n * n * bpe / (ms / 1e3) / 1e9
        return {"ms": ms, "gbs": gbs, "frac": gbs / peak, "bytes_per_elem": bpe, "yardstick": yard,
                "yardstick_ms": yard_ms, "vs_yardstick": ms / yard_ms}

    res = {"n": n}
    t = torch.empty((n, n), dtype=torch.int32, device="cuda")
    out = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(t, 1451, "u8")
    img = t.to(torch.uint8)
    cp5 = med(lambda: out.copy_(img))
    res["u8_integral_image"] = entry(med(lambda: sat.sat_u8(img, out=out)), 5, cp5, "u8 -> int32 copy_")
    res["batched_u8_16384x256x256"] = entry(med(lambda: sat.sat_batched_u8(img.view(-1, 256, 256),
                                                                            out=out.view(-1, 256, 256))),
                                            5, cp5, "u8 -> int32 copy_")
    del img
    satgen.fill_tensor(t, 1447, "u32")
    cp8 = med(lambda: out.copy_(t))
    res["batched_i32_16384x256x256"] = entry(med(lambda: sat.sat_batched(t.view(-1, 256, 256),
                                                                         out=out.view(-1, 256, 256))),
                                             8, cp8, "int32 copy_")
    res["box_sum_r8"] = entry(med(lambda: sat.box_sum(t, 8, 8, out=out)), 8, cp8, "int32 copy_")
    res["box_sum_r64"] = entry(med(lambda: sat.box_sum(t, 64, 64, out=out)), 8, cp8, "int32 copy_")
    del out
    satgen.fill_tensor(t, 1447, "f01")
    xf = t.view(torch.float32)
    y64 = torch.empty((n, n), dtype=torch.float64, device="cuda")
    cp12 = med(lambda: y64.copy_(xf))
    res["f32_f64_sat"] = entry(med(lambda: sat.sat_f64(xf, out=y64)), 12, cp12, "fp32 -> fp64 copy_")
    ym = y64.view(torch.float32).view(n, n, 2)
    res["moments_f32"] = entry(med(lambda: sat.sat_moments(xf, out=ym)), 12, cp12, "fp32 -> fp64 copy_")
    del t, xf, y64, ym
    torch.cuda.empty_cache()
    return res


def chain_projection(torch, sat, satgen, n, single_ms) -> dict:
    """configs[4] (64K^2 int32 strips on N GPUs) with the chained partition, emulated on this one GPU:
    * per_rank_ms: every rank's kernel alone on the whole GPU, ranks one after the other on one stream
      (each finds its upstream column sums already in its inbox): the per-GPU work of an N-GPU run;
      projected efficiency = single-pass 64K^2 time / (N * slowest rank), i.e. linear scaling minus the
      per-rank overheads (the start-up lag of one tile column and NVLink latency are not in it);
    * concurrent_ms: all N ranks' kernels at once on N streams, the GPU's SMs split N ways, the whole
      in-kernel protocol (pushes, inbox waits, back-pressure) running; efficiency = single / concurrent.
    In place on one 16 GiB matrix (timings do not depend on the values)."""
    res = {"single_pass_ms": single_ms}
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, 1447, "u32")
    sms = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
    for N in (2, 4, 8):
        h = n // N
        parts = [x[r * h:(r + 1) * h] for r in range(N)]
        chains = sat.Chain.local(N, n)
        try:
            per = [0.0] * N
            for it in range(4):
                evs = [torch.cuda.Event(enable_timing=True) for _ in range(N + 1)]
                evs[0].record()
                for r in range(N):
                    sat.sat_chained(parts[r], out=parts[r], chain=chains[r])
                    evs[r + 1].record()
                torch.cuda.synchronize()
                if it > 0:
                    per = [max(per[r], evs[r].elapsed_time(evs[r + 1])) if it > 1 else evs[r].elapsed_time(evs[r + 1])
                           for r in range(N)]
            streams = [torch.cuda.Stream() for _ in range(N)]
            sat.set_max_ctas(sms // N)
            try:
                times = []
                for it in range(4):
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    for st in streams:
                        st.wait_event(e0)
                    for r in range(N):
                        sat.sat_chained(parts[r], out=parts[r], chain=chains[r], stream=streams[r])
                    for st in streams:
                        torch.cuda.current_stream().wait_stream(st)
                    e1.record()
                    torch.cuda.synchronize()
                    if it > 0:
                        times.append(e0.elapsed_time(e1))
            finally:
                sat.set_max_ctas(0)
            slowest = max(per)
            conc = min(times)
            res[str(N)] = {"per_rank_ms": per, "slowest_rank_ms": slowest,
                           "projected_efficiency": single_ms / (N * slowest),
                           "concurrent_ms": conc, "concurrent_efficiency": single_ms / conc,
                           "gather_path_note": "colsum + all-gather + SAT reads each element twice: <= ~0.67"}
        finally:
            for c in chains:
                c.close()
    del x
    torch.cuda.empty_cache()
    return res


def run_sweep(args, sat, satgen, torch):
    """Table III analogue: n = 256 .. 32K, SAT vs same-run memcpy, overhead %."""
    dev = torch.device("cuda", torch.cuda.current_device())
    tdt = torch.float32 if args.dtype == "f32" else torch.int32
    stream = torch.cuda.current_stream()
    for k in range(8, 16):
        n = 1 << k
        x = torch.empty((n, n), dtype=torch.int32, device=dev)
        satgen.fill_tensor(x, 1447, "f01" if args.dtype == "f32" else "u32")
        x = x.view(tdt)
        y = torch.empty_like(x)
        reps = max(args.steps, int(2e9 / (n * n * 8)))
        reps = min(reps, 2000)

        def timeit(fn):
            for _ in range(max(3, args.warmup)):
                fn()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            for _ in range(reps):
                fn()
            b.record(stream)
            torch.cuda.synchronize()
            return a.elapsed_time(b) / reps

        t_sat = timeit(lambda: sat.sat(x, out=y))
        t_cp = timeit(lambda: y.copy_(x))
        print(json.dumps({"n": n, "dtype": args.dtype, "sat_ms": t_sat, "memcpy_ms": t_cp,
                          "overhead_pct": (t_sat - t_cp) / t_cp * 100, "sat_gelems": n * n / t_sat / 1e6,
                          "sat_gbs": n * n * 8 / t_sat / 1e6, "memcpy_gbs": n * n * 8 / t_cp / 1e6,
                          "reps": reps}), flush=True)
        del x, y
    return 0


if __name__ == "__main__":
    sys.exit(main())
