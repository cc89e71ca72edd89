"""One fp32 -> fp64 SAT launch at 32K x 32K after warm-ups, for an ncu capture."""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

n = 32768
x = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01")
x = x.view(torch.float32)
y = torch.empty((n, n), dtype=torch.float64, device="cuda")
for _ in range(4):
    sat.sat_f64(x, out=y)
torch.cuda.synchronize()
print("done")
