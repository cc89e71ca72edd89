"""Box filter (NEXT-4) device time at n x n int32 for a few radii vs the same-run int32 copy
(4 B read + 4 B written per element).  python tools/bench_box.py [n]"""
import json
import statistics
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402


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


n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
t = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(t, 1447, "u32")
out = torch.empty_like(t)
cp = med(lambda: out.copy_(t))
for rh, rw in [(1, 1), (8, 8), (32, 32), (64, 64), (8, 200), (100, 8)]:
    ms = med(lambda: sat.box_sum(t, rh, rw, out=out))
    print(json.dumps({"n": n, "rh": rh, "rw": rw, "ms": round(ms, 4), "gbs": round(n * n * 8 / ms / 1e6, 1),
                      "copy_ms": round(cp, 4), "vs_copy": round(ms / cp, 3)}), flush=True)
