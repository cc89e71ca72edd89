"""Raw per-tile timeline of one SAT launch (instrumented build libsat_stats.so) saved for offline analysis:
gpurun_out/trace_<n>_<variant>.npz with trace[ntiles, 8] (%globaltimer ns: 0 acquired, 1 data landed,
2 local aggregates published, 3 row walk resolved, 4 column walk resolved, 5 Step 4 done, 6 store issued,
7 TMA load issued), the tile grid, and the device time of an uninstrumented-sized launch.
python tools/trace_dump.py --n 4096 --variant 1"""
import argparse
import ctypes
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

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=4096)
ap.add_argument("--variant", type=int, default=-1)
ap.add_argument("--order", type=int, default=0)
a = ap.parse_args()
sat.set_tuning(a.variant, a.order, 0)
x = torch.empty((a.n, a.n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "u32")
y = torch.empty_like(x)
for _ in range(3):
    sat.sat(x, out=y)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
sat.sat(x, out=y)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1)
plan = sat.query_plan(0, a.n, a.n, a.n, x.data_ptr(), y.data_ptr())
nt = plan["tiles"]
buf = np.zeros(8 * nt, dtype=np.int64)
n = ctypes.c_int64()
_lib.check(_lib.lib().sat_debug_trace(buf.ctypes.data, nt, ctypes.byref(n)), "trace")
Path("gpurun_out").mkdir(exist_ok=True)
out = f"gpurun_out/trace_{a.n}_{plan['variant']}_{a.order}.npz"
np.savez_compressed(out, trace=buf.reshape(nt, 8), TR=plan["tile_rows"], TC=plan["tile_cols"], n=a.n, ms=ms,
                    order=plan["order"], ctas=plan["ctas"])
print(out, "ms", ms, "tiles", nt, "ctas", plan["ctas"])
