"""Rebuild libsat.so (or the stats build with --stats) and print registers / spills per kernel."""
import re
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import build_native  # noqa: E402

extra = ["-DSAT_STATS=1"] if "--stats" in sys.argv else []
out = ROOT / "paper_conf_ipps_emotofthni18_b200" / ("libsat_stats.so" if extra else "libsat.so")
inc = ["-I", str(ROOT / "include"), "-I", str(build_native.CSRC)]
nccl = build_native._nccl_include()
if nccl:
    inc += ["-I", nccl, "-DSAT_HAVE_NCCL_H=1"]
cmd = [build_native.NVCC, *build_native.ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xptxas", "-v", "-Xcompiler",
       "-fPIC,-fvisibility=hidden", "-shared", "--cudart", "shared", *inc, *extra,
       *[str(s) for s in sorted(build_native.CSRC.glob("*.cu"))], "-o", str(out), "-ldl"]
log = subprocess.run(cmd, capture_output=True, text=True).stderr
name = None
for line in log.splitlines():
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        name = subprocess.run(["c++filt", m.group(1)], capture_output=True, text=True).stdout.strip()
        name = name.replace("sat::", "").replace("unsigned int", "u32")
    m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and name:
        spill = f"spill {m.group(1)}/{m.group(2)}"
    m = re.search(r"Used (\d+) registers", line)
    if m and name:
        print(f"{m.group(1):>4} regs  {spill:<16} {name[:150]}")
        name = None
