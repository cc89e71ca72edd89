"""Per-role cycle breakdown of the warp-specialised SAT kernel (instrumented build libsat_stats.so).
Usage: python tools/stats_ws.py [--n 32768] [--variants 0,1]"""
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

NAMES = ["tiles", "c_full_wait", "c_local", "c_walk_wait", "c_finish", "row_rounds", "col_rounds",
         "st_result_wait", "st_store", "ld_issue", "ld_empty_wait", "c_bandbar", "row_tiles", "col_tiles",
         "row_round_cyc", "col_round_cyc", "row_resolve", "col_resolve", "row_idle_rounds", "col_idle_rounds",
         "row_load_lat", "col_load_lat", "fast_hits", "c_scan"]
ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--variants", default="0,1")
ap.add_argument("--dtype", default="f32")
ap.add_argument("--order", type=int, default=0)
a = ap.parse_args()
x = torch.empty((a.n, a.n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01" if a.dtype == "f32" else "u32")
if a.dtype == "f32":
    x = x.view(torch.float32)
y = torch.empty_like(x)
for v in [int(s) for s in a.variants.split(",")]:
    sat.set_tuning(v, a.order, 0)
    for _ in range(3):
        sat.sat(x, out=y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    sat.sat(x, out=y)
    e1.record()
    torch.cuda.synchronize()
    buf = np.zeros((4096, 24), dtype=np.int64)
    nc, ns = ctypes.c_int(), ctypes.c_int()
    _lib.check(_lib.lib().sat_debug_stats(buf.ctypes.data, 4096, ctypes.byref(nc), ctypes.byref(ns)), "stats")
    st = buf[: nc.value]
    tiles = st[:, 0].sum()
    print(json.dumps({"variant": v, "ms": round(e0.elapsed_time(e1), 4), "ctas": int(nc.value), "tiles": int(tiles),
                      "per_tile": {NAMES[k]: round(float(st[:, k].sum()) / tiles, 1) for k in range(1, 24)}}),
          flush=True)
