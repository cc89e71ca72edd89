"""Poll latency while the SAT kernel itself saturates HBM (probe block co-resident with SAT CTAs)."""
import ctypes, sys
from pathlib import Path
sys.path.insert(0, str(Path(__file__).resolve().parents[2]))
import torch
import paper_conf_ipps_emotofthni18_b200 as sat
import satgen
lib = ctypes.CDLL(str(Path(__file__).resolve().parent / "liblatprobe.so"))
n = 32768
x = torch.empty((n, n), dtype=torch.int32, device="cuda"); satgen.fill_tensor(x, 1, "f01"); x = x.view(torch.float32)
y = torch.empty_like(x)
flags = torch.zeros(4096 * 16, dtype=torch.int64, device="cuda")
out = torch.zeros(4, dtype=torch.int64, device="cuda")
s2 = torch.cuda.Stream()
for v in [0, 5]:
    sat.set_tuning(v, 0, 0)
    sat.sat(x, out=y); torch.cuda.synchronize()
    lib.probe_async(ctypes.c_void_p(flags.data_ptr()), 200, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s2.cuda_stream))
    torch.cuda.synchronize(); idle = int(out[0])
    for rep in range(3):
        sat.sat(x, out=y)
        with torch.cuda.stream(s2):
            lib.probe_async(ctypes.c_void_p(flags.data_ptr()), 3000, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s2.cuda_stream))
        torch.cuda.synchronize()
        print(f"variant {v}: idle {idle} cyc, during SAT {int(out[0])} cyc")
