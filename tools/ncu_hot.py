"""Top stalled SASS instructions of an ncu report (address, opcode, executed, stall share).
usage: python tools/ncu_hot.py report.ncu-rep [n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 60
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]
data = [dict(zip(h, r)) for r in rows[2:]]
tot = sum(float(d["Warp Stall Sampling (All Samples)"] or 0) for d in data)
keys = [k for k in h if k.startswith("stall_") or "Stall" in k]
data.sort(key=lambda d: -float(d["Warp Stall Sampling (All Samples)"] or 0))
for d in data[:n]:
    s = float(d["Warp Stall Sampling (All Samples)"] or 0)
    print("%6s %-60s %10s %5.1f%%" % (d.get("Address", "?"), d["Source"].strip()[:60], d["Instructions Executed"],
                                      100 * s / tot))
