"""Per-tile timeline of one SAT launch (libsat_stats.so): completion rate over time and the tile
latency (acquisition -> store) by anti-diagonal.  python tools/trace_ws.py [--variant V]"""
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

import oracle  # noqa: E402  (the Fig. 9 order, to map serials to diagonals)
import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
from paper_conf_ipps_emotofthni18_b200 import _lib  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--variant", type=int, default=0)
a = ap.parse_args()
sat.set_tuning(a.variant, 0, 0)
x = torch.empty((a.n, a.n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01")
x = x.view(torch.float32)
y = torch.empty_like(x)
for _ in range(3):
    sat.sat(x, out=y)
torch.cuda.synchronize()
plan = sat.query_plan(1, a.n, a.n, a.n, x.data_ptr(), y.data_ptr())
nt = plan["tiles"]
buf = np.zeros(8 * nt, dtype=np.int64)
n = ctypes.c_int64()
_lib.check(_lib.lib().sat_debug_trace(buf.ctypes.data, nt, ctypes.byref(n)), "trace")
acq, done = buf[0::8].astype(np.float64), buf[6::8].astype(np.float64)  # acquired, store issued
t0 = acq.min()
acq -= t0
done -= t0
R, C = -(-a.n // plan["tile_rows"]), -(-a.n // plan["tile_cols"])
diag = np.array([I + J for I, J in oracle.tile_order(R, C)])
lat = done - acq
end = done.max()
bins = np.linspace(0, end, 21)
hist, _ = np.histogram(done, bins)
out = {"variant": a.variant, "tiles": int(nt), "span_us": end / 1e3,
       "completed_per_5pct": hist.tolist(),
       "lat_us_by_diag_decile": [], "mean_lat_us": float(lat.mean() / 1e3)}
dmax = diag.max()
for q in range(10):
    sel = (diag >= q * (dmax + 1) / 10) & (diag < (q + 1) * (dmax + 1) / 10)
    out["lat_us_by_diag_decile"].append(round(float(lat[sel].mean() / 1e3), 2))
# time at which each decile of the serial order completes
order = np.argsort(np.arange(nt))
out["serial_decile_done_us"] = [round(float(np.percentile(done[i * nt // 10:(i + 1) * nt // 10], 50) / 1e3), 1)
                                for i in range(10)]
print(json.dumps(out))
