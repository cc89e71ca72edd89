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
def cpu_oracle_sample(rows: int, cols: int, dtype: str, target_s: float = 12.0) -> dict:
    """Time the CPU oracle (oracle/, as it stands, single thread) on a bounded sample of the workload:
    the first `h` rows (all columns) of the same seeded matrix, h chosen for ~target_s of CPU work."""
    import numpy as np

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

    h = min(rows, 64)
    t = run(h)
    while t < 0.5 and h < rows:
        h = min(rows, h * 4)
        t = run(h)
    rate = h * cols / t
    h2 = int(min(rows, max(h, rate * target_s / cols)))
    if h2 > h:
        h, t = h2, run(h2)
    return {"value": h * cols / t / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"first {h} of {rows} rows x {cols} cols ({dtype}, seed 1447), in-memory oracle "
                      f"(column-then-row, single thread), {t:.2f} s", "_np": np.__version__}


# ------------------------------------------------------------------------------------- helpers
def order_name(order: int) -> str:
    """Tile order of the plan: 0 anti-diagonal (Fig. 9), 1 row-major, (g << 8) diagonal of g-tile groups."""
    g = (order >> 8) & 255
    if (order & 15) == 0 and g > 1:
        return f"anti-diagonal of {g}-tile groups"
    return ["anti-diagonal", "row-major"][order & 15]


def load_ncu_traffic(workload: str):
    p = ROOT / "profiles" / "ncu_summary.json"
    if not p.exists():
        return None
    try:
        d = json.loads(p.read_text())
        e = d.get(workload)
        return None if e is None else e.get("dram_bytes_per_launch")
    except Exception:
        return None


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
    for _ in range(args.warmup):
        f()
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        f()
        times.append(time.perf_counter() - t0)
    ms = statistics.mean(times) * 1e3
    value = h * cols / (ms / 1e3) / 1e9
    sample = f"first {h} of {rows} rows x {cols} cols per step ({dtype}, seed 1447), single-thread C oracle"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak" if world == 1 else "strong",
        "vs_baseline": None, "dtype": "f64" if dtype == "f32" else "u32", "data": "synthetic",
        "config": {"workload": f"{n}x{n} {dtype} SAT (sampled rows)", "rows": rows, "cols": cols},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
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
    comm = sat.Comm() if world > 1 else None

    def step():
        if comm is None:
            sat.sat(x, out=y)
        else:
            sat.sat_sharded(x, out=y, comm=comm)

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
    sat.sat(x, out=y) if comm is None else sat.sat_sharded(x, out=y, comm=comm)
    torch.cuda.synchronize()

    # ---- end to end through the C ABI with host buffers (rank 0 of N=1 only; PCIe-bound)
    e2e = None
    if rank == 0 and world == 1 and not args.no_e2e:
        h_in = torch.empty((rows, cols), dtype=tdt, pin_memory=True)
        h_out = torch.empty((rows, cols), dtype=tdt, pin_memory=True)
        h_in.copy_(x)
        sat.sat_host(h_in.numpy(), h_out.numpy())  # warm-up (allocates the staging buffer)
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            sat.sat_host(h_in.numpy(), h_out.numpy())
        e2e_s = (time.perf_counter() - t0) / args.e2e_steps
        ok = bool(torch.equal(h_out[-1, -8:].to(dev), y[-1, -8:])) if args.dtype == "i32" else True
        e2e = {"value": total_elems / e2e_s / 1e9, "unit": UNIT, "h2d_bytes_per_step": total_elems * 4,
               "d2h_bytes_per_step": total_elems * 4, "ms_per_step": e2e_s * 1e3,
               "path": "sat_compute_host (pinned host buffers; strip-pipelined H2D | SAT | D2H)", "check": ok}
        del h_in, h_out

    if rank == 0:
        peak, peak_src = measured_peaks()
        kernel_ms = ms  # one SAT launch per step (N=1)
        achieved = (nrows * cols * BYTES_PER_ELEM) / (kernel_ms / 1e3) / 1e9
        workload = f"{n}x{n} {args.dtype} SAT" + ("" if world == 1 else f" strip-partitioned over {world} GPUs")
        plan = sat.query_plan(sat.SAT_FLOAT32 if args.dtype == "f32" else sat.SAT_INT32, nrows, cols, cols,
                              x.data_ptr(), y.data_ptr())
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
                       "parallelism": "single GPU" if world == 1 else f"strips x{world}"},
            "hbm_gbs": achieved,
            "memcpy": {"ms": memcpy_ms, "gbs": nrows * cols * BYTES_PER_ELEM / (memcpy_ms / 1e3) / 1e9,
                       "overhead_pct": (ms - memcpy_ms) / memcpy_ms * 100.0},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": load_ncu_traffic(workload), "peak_source": peak_src,
                         "kernel": {2: "sat_tm_kernel", 1: "sat_ws_kernel"}.get(plan["family"], "sat_tiles_kernel"),
                         "bytes_per_elem": BYTES_PER_ELEM},
            "gpu_launches": args.steps * (1 if world == 1 else 4),
            "clocks": clk,
            "e2e": e2e,
        }
        if world == 1 and not args.no_cpu:
            cb = cpu_oracle_sample(rows, cols, args.dtype)
            cb.pop("_np", None)
            line["cpu_baseline"] = cb
        print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
        dist.destroy_process_group()
    return 0


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
