"""Sweep kernel variants / tile orders / CTAs per SM at one matrix size (tuning aid, not the bench).
Prints one JSON line per configuration: SAT ms, memcpy ms, overhead %."""
import argparse
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--dtype", default="f32")
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--variants", default="all")
ap.add_argument("--orders", default="0,1")
ap.add_argument("--ctas", default="0")
a = ap.parse_args()
n = a.n
x = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01" if a.dtype == "f32" else "u32")
if a.dtype == "f32":
    x = x.view(torch.float32)
y = torch.empty_like(x)


def timeit(fn, reps):
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


cp = timeit(lambda: y.copy_(x), a.reps)
variants = range(sat.num_variants()) if a.variants == "all" else [int(v) for v in a.variants.split(",")]
ref = None
for v in variants:
    for order in [int(o) for o in a.orders.split(",")]:
        for c in [int(c) for c in a.ctas.split(",")]:
            sat.set_tuning(v, order, c)
            ms = timeit(lambda: sat.sat(x, out=y), a.reps)
            if a.dtype != "f32":
                if ref is None:
                    ref = y.clone()
                ok = bool(torch.equal(ref, y))
            else:
                ok = None
            plan = sat.query_plan(1 if a.dtype == "f32" else 0, n, n, n, x.data_ptr(), y.data_ptr())
            print(json.dumps({"n": n, "variant": v, "tile": [plan["tile_rows"], plan["tile_cols"]], "order": order,
                              "ctas_per_sm": c, "ctas": plan["ctas"], "sat_ms": round(ms, 4), "memcpy_ms": round(cp, 4),
                              "overhead_pct": round((ms - cp) / cp * 100, 1), "gbs": round(n * n * 8 / ms / 1e6, 1),
                              "same_as_first": ok}), flush=True)
sat.set_tuning(-1, 0, 0)
