"""configs[4] chained-partition projection on one GPU (bench.chain_projection) without the rest of the bench."""
import json
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

n = 65536
x = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "u32")
single = bench.event_time(torch, lambda: sat.sat(x, out=x), 5)
del x
torch.cuda.empty_cache()
res = bench.chain_projection(torch, sat, satgen, n, single)
for N in ("2", "4", "8"):
    r = res[N]
    print(N, " ".join(f"{v:.3f}" for v in r["per_rank_ms"]), f"proj {r['projected_efficiency']:.3f}",
          f"conc {r['concurrent_ms']:.3f} ({r['concurrent_efficiency']:.3f})")
print(json.dumps(res))
