"""Top source lines by warp-stall samples from an ncu report (cuda,sass source page), with the
dominant stall reasons.  python tools/ncu_lines.py REPORT.ncu-rep [TOP]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, fname, header = [], None, None
for rec in csv.reader(io.StringIO(txt)):
    if not rec:
        continue
    if rec[0] in ("File Name", "File Path"):
        fname = rec[1].split("/")[-1]
        continue
    if rec[0] == "Line No":
        header = rec
        continue
    if header and len(rec) == len(header) and rec[0].isdigit():
        i = header.index("Warp Stall Sampling (All Samples)")
        try:
            samp = int(rec[i])
        except ValueError:
            continue
        stalls = {k[6:]: int(v) for k, v in zip(header, rec) if k.startswith("stall_") and v.isdigit() and int(v) > 0}
        rows.append((samp, fname, int(rec[0]), rec[1].strip()[:70], stalls, ""))
tot = sum(r[0] for r in rows)
print("total samples", tot)
for samp, f, ln, src, stalls, ie in sorted(rows, reverse=True)[:top]:
    st = ", ".join(f"{k}:{v}" for k, v in sorted(stalls.items(), key=lambda kv: -kv[1])[:3])
    print(f"{100.0 * samp / tot:5.1f}% {f}:{ln:<4} {src:<70} | {st}")
