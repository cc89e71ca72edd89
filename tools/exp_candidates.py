"""Round-2 candidate configurations in the tuning build (SAT_LIB=.../libsat_exp.so): u8 integral image at 32K^2
per variant, and the chained 64K^2 strip per-rank time at N=8 per chain variant.
python tools/exp_candidates.py --u8 2,12 --chain 4,13,14"""
import argparse
import json
import os
import statistics
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
os.environ.setdefault("SAT_LIB", str(ROOT / "paper_conf_ipps_emotofthni18_b200" / "libsat_exp.so"))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--u8", default="")
ap.add_argument("--chain", default="")
a = ap.parse_args()


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


if a.u8:
    n = 32768
    t = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(t, 1451, "u8")
    img = t.to(torch.uint8)
    for v in [int(x) for x in a.u8.split(",")]:
        sat.set_tuning(v, 0, 0)
        ms = med(lambda: sat.sat_u8(img, out=t))
        print(json.dumps({"u8_variant": v, "ms": round(ms, 4), "gbs": round(n * n * 5 / ms / 1e6, 1)}), flush=True)
    sat.set_tuning(-1, 0, 0)
    del t, img
    torch.cuda.empty_cache()
if a.chain:
    n, N = 65536, 8
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, 1447, "u32")
    h = n // N
    parts = [x[r * h:(r + 1) * h] for r in range(N)]
    for v in [int(c) for c in a.chain.split(",")]:
        sat.set_tuning(v, 0, 0)
        chains = sat.Chain.local(N, n)
        per = []
        for it in range(4):
            evs = [torch.cuda.Event(enable_timing=True) for _ in range(N + 1)]
            evs[0].record()
            for r in range(N):
                sat.sat_chained(parts[r], out=parts[r], chain=chains[r])
                evs[r + 1].record()
            torch.cuda.synchronize()
            if it > 0:
                per.append(max(evs[r].elapsed_time(evs[r + 1]) for r in range(N)))
        for c in chains:
            c.close()
        print(json.dumps({"chain_variant": v, "slowest_rank_ms": round(min(per), 4)}), flush=True)
    sat.set_tuning(-1, 0, 0)
