"""Classic kernel (variant 0) forced at sizes with more tiles than resident CTAs, under CTA caps:
which configurations of the multi-tile persistent loop complete (tuning / debugging aid)."""
import os
import sys
import time

sys.path.insert(0, os.getcwd())
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

n = int(sys.argv[1])
caps = [int(c) for c in sys.argv[2].split(",")]
sat.set_tuning(0, 0, 0)
a = satgen.gen_host(n, n, seed=5, dist="u32")
want = oracle.sat_i32(a)
x = torch.from_numpy(a).cuda()
for cap in caps:
    sat.set_max_ctas(cap)
    for rep in range(3):
        t = time.time()
        got = sat.sat(x).cpu().numpy()
        print(sat._lib.LIB_PATH.name, "n", n, "cap", cap, "rep", rep, "ok", bool((got == want).all()),
              "%.3fs" % (time.time() - t), flush=True)
