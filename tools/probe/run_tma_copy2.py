"""Tile-shape / stage / data-path sweep of the TMA copy pipeline (tools/probe/tma_copy2.cu)."""
import ctypes
import sys
from pathlib import Path

import torch

lib = ctypes.CDLL(str(Path(__file__).resolve().parent / "libtmacopy2.so"))
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
print(f"torch copy_: {e0.elapsed_time(e1) / 10:.4f} ms", flush=True)
CFGS = [(128, 128, 2), (128, 128, 3), (64, 256, 3), (32, 512, 3)] if len(sys.argv) > 4 else [(128, 128, 2), (64, 256, 2), (32, 512, 2), (16, 1024, 2), (128, 128, 3), (64, 256, 3), (32, 512, 3),
        (16, 1024, 3), (32, 256, 4), (32, 256, 6), (16, 512, 4), (16, 512, 6), (64, 512, 1), (32, 1024, 1),
        (32, 1024, 2), (16, 2048, 2), (32, 128, 4), (64, 128, 4)]
modes = [int(m) for m in (sys.argv[2] if len(sys.argv) > 2 else "0,1").split(",")]
orders = [int(m) for m in (sys.argv[3] if len(sys.argv) > 3 else "0,1").split(",")]
for mode in modes:
    for order in orders:
        for tr, tc, st in CFGS:
            for promo in (2,):
                ms, lat = ctypes.c_float(), ctypes.c_double()
                rc = lib.tma_copy2(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(y.data_ptr()), n, tr, tc, st, mode,
                                   148, 10, order, promo, ctypes.byref(ms), ctypes.byref(lat))
                ok = bool(torch.equal(x, y)) if rc == 0 else False
                y.zero_()
                print(f"mode={mode} order={order} tr={tr} tc={tc} st={st} promo={promo}: rc={rc} {ms.value:.4f} ms "
                      f"{2 * 4 * n * n / max(ms.value, 1e-9) / 1e6:.0f} GB/s load_lat={lat.value / 1965:.2f} us ok={ok}",
                      flush=True)
