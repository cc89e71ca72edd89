"""TMA tile-pipeline copy probe (tools/probe/tma_copy.cu): time and mean load latency per config."""
import ctypes
import sys
from pathlib import Path

import torch

lib = ctypes.CDLL(str(Path(__file__).resolve().parent / "libtmacopy.so"))
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
x = torch.rand((n, n), device="cuda")
y = torch.empty_like(x)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(3):
    y.copy_(x)
e0.record()
for _ in range(10):
    y.copy_(x)
e1.record()
torch.cuda.synchronize()
print(f"torch copy_: {e0.elapsed_time(e1) / 10:.4f} ms")
for blocks, unroll in [(148 * 4, 0), (148 * 4, 1), (148 * 8, 0), (148 * 2, 1), (148, 1)]:
    ms = ctypes.c_float()
    rc = lib.ldg_copy_run(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), ctypes.c_longlong(n * n), blocks,
                          unroll, 10, ctypes.byref(ms))
    print(f"ldg copy blocks={blocks} unroll={unroll}: rc={rc} {ms.value:.4f} ms {2 * 4 * n * n / ms.value / 1e6:.0f} GB/s",
          flush=True)
CFGS = [(128, 2, 148, 0, 128), (128, 2, 148, 2, 128), (64, 2, 148, 0, 256), (64, 2, 148, 2, 256),
        (64, 3, 148, 2, 256), (32, 4, 148, 2, 256), (64, 2, 296, 2, 256), (32, 3, 296, 2, 256)]
for tr, st, ctas, split, tc in CFGS:
    ms, lat = ctypes.c_float(), ctypes.c_double()
    rc = lib.tma_copy(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), n, tr, st, ctas, 10, split,
                      ctypes.byref(ms), ctypes.byref(lat), tc)
    ok = bool(torch.equal(x, y)) if rc == 0 else False
    y.zero_()
    print(f"tc={tc} tr={tr} stages={st} ctas={ctas} split={split}: rc={rc} {ms.value:.4f} ms "
          f"{2 * 4 * n * n / ms.value / 1e6:.0f} GB/s  load_lat={lat.value / 1920:.2f} us  ok={ok}", flush=True)
