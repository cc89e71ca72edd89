import ctypes, sys
from pathlib import Path
lib = ctypes.CDLL(str(Path(__file__).resolve().parent / "liblatprobe.so"))
for sms in [147, 74, 16]:
    idle, loaded, ms = ctypes.c_longlong(), ctypes.c_longlong(), ctypes.c_float()
    r = lib.run_probe(sms, 4, ctypes.byref(idle), ctypes.byref(loaded), ctypes.byref(ms))
    gbs = 4 * 2 * (1 << 32) / (ms.value / 1e3) / 1e9
    print(f"load_sms={sms} rc={r} idle_lat={idle.value} cyc loaded_lat={loaded.value} cyc copy={ms.value:.2f} ms ({gbs:.0f} GB/s)")
