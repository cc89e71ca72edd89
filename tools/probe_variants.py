import sys, os, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle, satgen
import paper_conf_ipps_emotofthni18_b200 as sat
print(sat._lib.LIB_PATH.name, flush=True)
for vi in [int(v) for v in sys.argv[1].split(",")]:
    sat.set_tuning(vi, 0, 0)
    for n in [int(v) for v in sys.argv[2].split(",")]:
        a = satgen.gen_host(n, n, seed=5, dist="u32")
        t = time.time()
        got = sat.sat(torch.from_numpy(a).cuda()).cpu().numpy()
        ok = (got == oracle.sat_i32(a)).all()
        print("variant", vi, "n", n, "ok", ok, "plan", sat.query_plan(0, n, n), "%.3fs" % (time.time() - t), flush=True)
