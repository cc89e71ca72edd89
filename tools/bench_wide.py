"""Device time of the 64-bit-element SATs (NEXT-3) at 16K x 16K vs a same-bytes copy (4 B read + 8 B written
per element): sat_compute_f32_f64 and sat_compute_moments_f32.  One JSON line per kernel."""
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402


def timeit(fn, reps=10):
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


n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
x = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01")
x = x.view(torch.float32)
y64 = torch.empty((n, n), dtype=torch.float64, device="cuda")
ym = torch.empty((n, n, 2), dtype=torch.float32, device="cuda")
# same-bytes yardstick: read n^2 fp32, write n^2 8-byte elements
cp = timeit(lambda: y64.view(torch.float32)[:, 0::2].copy_(x))
for name, fn in [("f32_f64", lambda: sat.sat_f64(x, out=y64)), ("moments_f32", lambda: sat.sat_moments(x, out=ym))]:
    ms = timeit(fn)
    gbs = n * n * 12 / ms / 1e6
    print(json.dumps({"kernel": name, "n": n, "sat_ms": round(ms, 4), "gbs_algorithmic": round(gbs, 1),
                      "bytes_per_elem": 12, "widen_copy_ms": round(cp, 4)}), flush=True)
