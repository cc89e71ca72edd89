"""Summarise one `ncu --set full` report of the SAT kernel into profiles/ncu_summary.json (the
`roofline.traffic` source of bench.py).  python tools/ncu_summary.py REPORT.ncu-rep WORKLOAD [OUT]"""
import csv
import io
import json
import subprocess
import sys
from pathlib import Path

rep, workload = sys.argv[1], sys.argv[2]
out = Path(sys.argv[3]) if len(sys.argv) > 3 else Path(__file__).resolve().parent.parent / "profiles" / "ncu_summary.json"
txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, units, vals = rows[0], rows[1], rows[2]  # one captured launch


def get(name, scale=1.0):
    i = hdr.index(name)
    v = float(vals[i].replace(",", ""))
    u = units[i]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-6, "usecond": 1e-3, "msecond": 1,
            "second": 1e3}.get(u, 1)
    return v * mult * scale


rd, wr = get("dram__bytes_read.sum"), get("dram__bytes_write.sum")
n = 32768 if "32768" in workload else None
summary = {
    "kernel": vals[hdr.index("Kernel Name")],
    "source": f"ncu --set full --clock-control none --import-source on ({Path(rep).name}), 1 launch after warm-ups",
    "gpu_time_ms": get("gpu__time_duration.sum"),
    "dram_bytes_read": rd,
    "dram_bytes_write": wr,
    "dram_bytes_per_launch": rd + wr,
    "algorithmic_bytes": 8 * n * n if n else None,
    "dram_over_algorithmic": (rd + wr) / (8 * n * n) if n else None,
    "dram_tbs": get("dram__bytes.sum.per_second") / (1e3 if units[hdr.index("dram__bytes.sum.per_second")] == "Gbyte/s" else 1),
    "dram_pct_of_peak": get("dram__bytes_read.sum.pct_of_peak_sustained_elapsed")
    + get("dram__bytes_write.sum.pct_of_peak_sustained_elapsed"),
    "sm_throughput_pct": get("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
    "issue_active_pct": get("sm__inst_issued.avg.pct_of_peak_sustained_active"),
    "inst_executed": get("smsp__inst_executed.sum"),
    "smem_per_block_kb": get("launch__shared_mem_per_block"),
    "l2_hit_rate_pct": get("lts__t_sector_hit_rate.pct"),
    "registers_per_thread": get("launch__registers_per_thread"),
    "grid": get("launch__grid_size"),
    "block": get("launch__block_size"),
}
doc = json.loads(out.read_text()) if out.exists() else {}
doc[workload] = summary
out.write_text(json.dumps(doc, indent=1) + "\n")
print(json.dumps(summary, indent=1))
