"""u8 integral-image kernel candidates (tuning aid): parity on small ragged images, then device time at
n x n for each (variant, order).  python tools/u8_probe.py N VARIANTS [ORDERS]"""
import os
import statistics
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402


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


n = int(sys.argv[1])
variants = [int(v) for v in sys.argv[2].split(",")]
orders = [int(o, 0) for o in sys.argv[3].split(",")] if len(sys.argv) > 3 else [0]
t = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(t, 1451, "u8")
img = t.to(torch.uint8)
for v in variants:
    for o in orders:
        sat.set_tuning(v, o, 0)
        for (r, c) in [(300, 517), (1000, 3001)]:
            im = satgen.gen_host(r, c, seed=7, dist="u8").astype(np.uint8)
            got = sat.sat_u8(torch.from_numpy(im).cuda()).cpu().numpy().view(np.uint32)
            assert (got == oracle.sat_u32(im.astype(np.uint32))).all(), (v, r, c)
        ms = med(lambda: sat.sat_u8(img, out=t))
        print("variant", v, "order", hex(o), "n", n, "ms", round(ms, 4), "GB/s", round(n * n * 5 / ms / 1e6, 1), flush=True)
sat.set_tuning(-1, 0, 0)
