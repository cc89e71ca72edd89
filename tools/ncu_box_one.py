"""One box filter launch at 32K x 32K int32 (radius argv[1]) after warm-ups, for an ncu capture."""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

r = int(sys.argv[1]) if len(sys.argv) > 1 else 8
n = 32768
t = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(t, 1447, "u32")
out = torch.empty_like(t)
for _ in range(4):
    sat.box_sum(t, r, r, out=out)
torch.cuda.synchronize()
print("done")
