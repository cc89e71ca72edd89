"""Device-time size sweep with CUDA graphs (host launch overhead excluded): SAT per variant vs D2D copy.
Usage: python tools/graph_sweep.py [--sizes 256,512,...] [--variants 0,4] [--dtype f32]"""
import argparse
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--sizes", default="256,512,1024,2048,4096,8192")
ap.add_argument("--variants", default="-1")
ap.add_argument("--dtype", default="f32")
ap.add_argument("--per-graph", type=int, default=20)
a = ap.parse_args()


def graph_time(fn, per_graph, reps=5):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(per_graph):
            fn()
    g.replay()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / per_graph)
    return best


for n in [int(s) for s in a.sizes.split(",")]:
    x = torch.empty((n, n), dtype=torch.int32, device="cuda")
    satgen.fill_tensor(x, 1447, "f01" if a.dtype == "f32" else "u32")
    if a.dtype == "f32":
        x = x.view(torch.float32)
    y = torch.empty_like(x)
    cp = graph_time(lambda: y.copy_(x), a.per_graph)
    for v in [int(s) for s in a.variants.split(",")]:
        sat.set_tuning(v, 0, 0)
        ms = graph_time(lambda: sat.sat(x, out=y), a.per_graph)
        print(json.dumps({"n": n, "variant": v, "sat_us": round(ms * 1e3, 2), "memcpy_us": round(cp * 1e3, 2),
                          "overhead_pct": round((ms - cp) / cp * 100, 1), "gbs": round(n * n * 8 / ms / 1e6, 1)}),
              flush=True)
    sat.set_tuning(-1, 0, 0)
