"""One sat_compute_batched launch per matrix shape at 2^30 int32 elements (for ncu: DRAM bytes and
duration of sat_batch_kernel).  python tools/batch_probe.py [--sizes 128,256,512,1024]"""
import argparse
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--sizes", default="128,256,512,1024")
args = ap.parse_args()
n = 32768
t = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(t, 1447, "u32")
out = torch.empty_like(t)
for s in (int(x) for x in args.sizes.split(",")):
    sat.sat_batched(t.view(-1, s, s), out=out.view(-1, s, s))
torch.cuda.synchronize()
