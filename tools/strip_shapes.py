"""SAT time of the per-rank strip shapes of the 64K x 64K strip-partitioned run (BASELINE configs[4]) on
one GPU: rows = 65536 / N, cols = 65536, int32, plus the strip column-sum pass.  One JSON line per N."""
import json
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
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return sorted(ts)[len(ts) // 2]


cols = 65536
for n in (8, 4, 2, 1):
    rows = 65536 // n
    if rows * cols * 8 > 60e9:
        continue
    x = torch.empty((rows, cols), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, 1447, "u32")
    y = torch.empty_like(x)
    t_sat = med(lambda: sat.sat(x, out=y))
    t_cs = med(lambda: sat.strip_colsum(x))
    t_cp = med(lambda: y.copy_(x))
    print(json.dumps({"ranks": n, "rows": rows, "cols": cols, "sat_ms": round(t_sat, 4), "colsum_ms": round(t_cs, 4),
                      "copy_ms": round(t_cp, 4), "sat_over_copy": round(t_sat / t_cp, 3),
                      "sat_gbs": round(rows * cols * 8 / t_sat / 1e6, 1)}), flush=True)
    del x, y
    torch.cuda.empty_cache()
