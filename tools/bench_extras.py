"""Throughput of the paths around the SAT hot path at 32K x 32K (one JSON line each):
u8 -> uint32 integral image (1 B read + 4 B written per element), box filter from a SAT (4 + 4 B),
int32 SAT.  CUDA events, warm-up 3, median of 10; inputs larger than L2.
python tools/bench_extras.py [--n 32768]"""
import argparse
import json
import statistics
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
a = ap.parse_args()
n = a.n


def med_ms(fn, reps=10):
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


def line(name, ms, bytes_per_elem, copy_ms):
    print(json.dumps({"path": name, "n": n, "ms": round(ms, 4), "gelems": round(n * n / ms / 1e6, 1),
                      "gbs": round(n * n * bytes_per_elem / ms / 1e6, 1), "bytes_per_elem": bytes_per_elem,
                      "same_bytes_copy_ms": round(copy_ms, 4), "overhead_pct": round((ms - copy_ms) / copy_ms * 100, 1)}),
          flush=True)


t = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(t, 1451, "u8")
img = t.to(torch.uint8)
out = torch.empty((n, n), dtype=torch.int32, device="cuda")
# yardstick for 5 B/elem: copy n*n*5/2 bytes each way is not a real op; use a u8->int32 widening copy (1 R + 4 W)
cp = med_ms(lambda: out.copy_(img))
line("u8_integral_image", med_ms(lambda: sat.sat_u8(img, out=out)), 5, cp)
del img
satgen.fill_tensor(t, 1447, "u32")
cp = med_ms(lambda: out.copy_(t))
line("i32_sat", med_ms(lambda: sat.sat(t, out=out)), 8, cp)
line("box_sum_r8", med_ms(lambda: sat.box_sum(t, 8, 8, out=out)), 8, cp)
line("box_sum_r64", med_ms(lambda: sat.box_sum(t, 64, 64, out=out)), 8, cp)
# batches of small matrices (sat_compute_batched, one launch) vs the same bytes copied, and vs one
# sat_compute launch per matrix (timed on the first 256 matrices, scaled to the batch)
for s in (128, 256, 512, 1024):
    tb = t.view(-1, s, s)
    ob = out.view(-1, s, s)
    ms = med_ms(lambda: sat.sat_batched(tb, out=ob))
    line(f"batched_{tb.shape[0]}x{s}x{s}_i32", ms, 8, cp)
    k = 256
    loop_ms = med_ms(lambda: [sat.sat(tb[i], out=ob[i]) for i in range(k)], reps=3) * tb.shape[0] / k
    print(json.dumps({"path": f"looped_single_{s}x{s}_i32", "ms_scaled": round(loop_ms, 3),
                      "batched_speedup": round(loop_ms / ms, 1)}), flush=True)
# batched u8 -> uint32 integral images (1 B read + 4 B written per pixel) vs the widening copy
img = t.to(torch.uint8)
cp5 = med_ms(lambda: out.copy_(img))
for s in (256, 1024):
    ms = med_ms(lambda: sat.sat_batched_u8(img.view(-1, s, s), out=out.view(-1, s, s)))
    line(f"batched_u8_{n * n // (s * s)}x{s}x{s}", ms, 5, cp5)
