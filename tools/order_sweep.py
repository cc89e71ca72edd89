import sys, os, json
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_emotofthni18_b200 as sat
import satgen
def graph_time(fn, per_graph=20, reps=5):
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3): fn()
    torch.cuda.current_stream().wait_stream(s); torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(per_graph): fn()
    g.replay(); torch.cuda.synchronize(); best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize(); best = min(best, e0.elapsed_time(e1) / per_graph)
    return best
for n in (4096, 8192):
    x = torch.empty((n, n), dtype=torch.int32, device="cuda"); satgen.fill_tensor(x, 1447, "u32"); y = torch.empty_like(x)
    for order in (0, 0x200, 0x400, 3 | 0x200, 3 | 0x400, 1, 2):
        sat.set_tuning(1, order, 0)
        us = graph_time(lambda: sat.sat(x, out=y)) * 1e3
        print(json.dumps({"n": n, "order": hex(order), "us": round(us, 2)}), flush=True)
    sat.set_tuning(-1, 0, 0)
