"""Per-phase cycle breakdown of the SAT kernel (instrumented build libsat_stats.so, -DSAT_STATS=1).
Usage: SAT_LIB=paper_conf_ipps_emotofthni18_b200/libsat_stats.so python tools/stats.py [--n 32768] [--variants 0,3]"""
import argparse
import ctypes
import json
import os
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
os.environ.setdefault("SAT_LIB", str(ROOT / "paper_conf_ipps_emotofthni18_b200" / "libsat_stats.so"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
from paper_conf_ipps_emotofthni18_b200 import _lib  # noqa: E402
import satgen  # noqa: E402

NAMES = ["tiles", "loop", "ticket", "full_wait", "compute", "row_lb", "row_steps", "row_spins", "col_lb",
         "col_steps", "col_spins", "diag_try", "diag_unresolved", "diag_late", "bar3_producer", "store",
         "store_wait", "bar1", "publish", "bar3"]

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--variants", default="0")
ap.add_argument("--orders", default="0")
ap.add_argument("--dtype", default="f32")
a = ap.parse_args()
x = torch.empty((a.n, a.n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01" if a.dtype == "f32" else "u32")
if a.dtype == "f32":
    x = x.view(torch.float32)
y = torch.empty_like(x)
for v in [int(s) for s in a.variants.split(",")]:
    for order in [int(s) for s in a.orders.split(",")]:
        sat.set_tuning(v, order, 0)
        for _ in range(3):
            sat.sat(x, out=y)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        sat.sat(x, out=y)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        buf = np.zeros((4096, len(NAMES)), dtype=np.int64)
        nc, ns = ctypes.c_int(), ctypes.c_int()
        _lib.check(_lib.lib().sat_debug_stats(buf.ctypes.data, 4096, ctypes.byref(nc), ctypes.byref(ns)), "stats")
        st = buf[: nc.value]
        tiles = st[:, 0].sum()
        per_tile = {NAMES[k]: round(float(st[:, k].sum()) / tiles, 1) for k in range(1, len(NAMES))}
        out = {"n": a.n, "variant": v, "order": order, "ms": round(ms, 4), "ctas": int(nc.value),
               "tiles": int(tiles), "tiles_per_cta_min": int(st[:, 0].min()), "tiles_per_cta_max": int(st[:, 0].max()),
               "per_tile_cycles": per_tile}
        print(json.dumps(out), flush=True)
