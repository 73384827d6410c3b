"""Summarise an ncu report: key SOL metrics + per-opcode instruction mix and stalls.
usage: python tools/ncu_summary.py report.ncu-rep [per_tile_divisor]"""
import collections
import csv
import io
import re
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
keep = {"Duration", "Elapsed Cycles", "SM Frequency", "Compute (SM) Throughput", "Issue Slots Busy",
        "Executed Ipc Active", "Issued Instructions", "Registers Per Thread", "Achieved Active Warps Per SM",
        "No Eligible", "Eligible Warps Per Scheduler", "Warp Cycles Per Issued Instruction", "DRAM Throughput",
        "Grid Size", "Block Size", "Dynamic Shared Memory Per Block"}
for r in rows[1:]:
    d = dict(zip(h, r))
    if d.get("Metric Name") in keep:
        print("%-40s %s %s" % (d["Metric Name"], d["Metric Value"], d["Metric Unit"]))
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
if len(rr) > 2:
    hh = rr[0]
    units = dict(zip(hh, rr[1]))
    vals = dict(zip(hh, rr[2]))
    for k in hh:
        if re.search(r"pipe_tensor.*active|dram__bytes_(read|write)\.sum$|sm__inst_executed_pipe_(alu|fma|fp16|uniform|xu).*sum$", k):
            print("%-70s %s %s" % (k, vals[k], units.get(k, "")))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"], capture_output=True,
                     text=True).stdout
srows = list(csv.reader(io.StringIO(src)))
hh = srows[1]
data = [dict(zip(hh, r)) for r in srows[2:]]
counts = sorted(float(d["Instructions Executed"] or 0) for d in data if float(d["Instructions Executed"] or 0) > 0)
div = float(sys.argv[2]) if len(sys.argv) > 2 else collections.Counter(counts).most_common(1)[0][0]
ops = collections.Counter()
st = collections.Counter()
tot = 0
for d in data:
    n = float(d["Instructions Executed"] or 0)
    s = float(d["Warp Stall Sampling (All Samples)"] or 0)
    op = re.sub(r"^@!?U?P\w+\s+", "", d["Source"].strip()).split(" ")[0]
    ops[op] += n / div
    st[op] += s
    tot += n
print("instructions per unit (divisor %.4g): %.1f" % (div, tot / div))
ts = sum(st.values())
for op, c in ops.most_common(40):
    print("%-30s %7.1f  stall %5.1f%%" % (op, c, 100 * st[op] / ts))
