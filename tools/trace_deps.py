"""Dependency timeline of one SAT launch (libsat_stats.so): for steady-state tiles, when did the row /
column walks resolve relative to the predecessors' local (LOCAL) and finish (INCL) publications?"""
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

import oracle  # noqa: E402
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
T = buf.reshape(nt, 8).astype(np.float64)
T[T == 0] = np.nan
T -= np.nanmin(T[:, 0])
R, C = -(-a.n // plan["tile_rows"]), -(-a.n // plan["tile_cols"])
order = oracle.tile_order(R, C)
serial = {ij: s for s, ij in enumerate(order)}
ACQ, LAND, LOC, ROWW, COLW, FIN, STO = range(7)
rows = []
for s, (I, J) in enumerate(order):
    if not (R // 4 <= I + J <= 3 * (R + C) // 4) or I == 0 or J == 0:
        continue
    L, U = serial[(I, J - 1)], serial[(I - 1, J)]
    rows.append([T[s, LAND] - T[s, ACQ], T[s, LOC] - T[s, ACQ], T[s, ROWW] - T[s, ACQ], T[s, COLW] - T[s, ACQ],
                 T[s, FIN] - T[s, ACQ], T[s, STO] - T[s, ACQ],
                 T[s, ROWW] - T[L, LOC], T[s, ROWW] - T[L, FIN], T[s, COLW] - T[U, LOC], T[s, COLW] - T[U, FIN],
                 T[L, LOC] - T[s, ACQ], T[L, FIN] - T[s, ACQ], T[s, LOC] - T[L, LOC], s - L, s - U])
A = np.array(rows)
names = ["land-acq", "local-acq", "roww-acq", "colw-acq", "fin-acq", "store-acq", "roww-L.local", "roww-L.fin",
         "colw-U.local", "colw-U.fin", "L.local-acq", "L.fin-acq", "local-L.local", "dserial_L", "dserial_U"]
print(json.dumps({"variant": a.variant, "steady_tiles": len(A),
                  "median_us": {k: round(float(np.nanmedian(A[:, i]) / 1e3), 2) for i, k in enumerate(names)},
                  "p90_us": {k: round(float(np.nanpercentile(A[:, i], 90) / 1e3), 2) for i, k in enumerate(names[:13])}}))

# walk wait of every interior tile: how long the compute warps sat between their local SAT and the later of
# the two walks, split by cause: predecessor INCL not yet published at local end (chain), or published but
# the walker had not caught it yet (poll latency)
waits, chain, poll, diags = [], [], [], []
for s, (I, J) in enumerate(order):
    if I == 0 or J == 0:
        continue
    L, U = serial[(I, J - 1)], serial[(I - 1, J)]
    walk = np.nanmax([T[s, ROWW], T[s, COLW]])
    w = max(0.0, walk - T[s, LOC])
    pred = np.nanmax([T[L, FIN], T[U, FIN]])
    c = max(0.0, min(walk, pred) - T[s, LOC])
    waits.append(w)
    chain.append(c)
    poll.append(w - c)
    diags.append(I + J)
waits, chain, poll, diags = map(np.array, (waits, chain, poll, diags))
dec = np.minimum((diags * 10) // (R + C - 1), 9)
LDI = 7
print(json.dumps({"load_latency_us_median": round(float(np.nanmedian(T[:, LAND] - T[:, LDI])) / 1e3, 2),
                  "load_latency_us_p90": round(float(np.nanpercentile(T[:, LAND] - T[:, LDI], 90)) / 1e3, 2),
                  "store_after_fin_us_median": round(float(np.nanmedian(T[:, STO] - T[:, FIN])) / 1e3, 2)}))
print(json.dumps({"mean_wait_us": round(float(np.nanmean(waits)) / 1e3, 3),
                  "mean_chain_us": round(float(np.nanmean(chain)) / 1e3, 3),
                  "mean_poll_us": round(float(np.nanmean(poll)) / 1e3, 3),
                  "frac_wait_gt_0.5us": round(float(np.mean(waits > 500)), 3),
                  "wait_by_diag_decile_us": [round(float(np.nanmean(waits[dec == q])) / 1e3, 2) for q in range(10)],
                  "chain_by_diag_decile_us": [round(float(np.nanmean(chain[dec == q])) / 1e3, 2) for q in range(10)]}))
