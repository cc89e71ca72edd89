"""Launch the SAT once (after warm-up) at n x n for ncu capture: python tools/ncu_one.py N DTYPE VARIANT REPS"""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

import paper_conf_ipps_emotofthni18_b200 as sat  # noqa: E402
import satgen  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
dtype = sys.argv[2] if len(sys.argv) > 2 else "f32"
variant = int(sys.argv[3]) if len(sys.argv) > 3 else -1
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 4
sat.set_tuning(variant, 0, 0)
x = torch.empty((n, n), dtype=torch.int32, device="cuda")
satgen.fill_tensor(x, 1447, "f01" if dtype == "f32" else "u32")
if dtype == "f32":
    x = x.view(torch.float32)
y = torch.empty_like(x)
for _ in range(reps):
    sat.sat(x, out=y)
torch.cuda.synchronize()
print("done", n, dtype, variant)
