"""Per-instruction stall breakdown of an ncu report (--page source, SASS view).

usage: python tools/ncu_source_stalls.py report.ncu-rep [kernel-regex] [top] [launch-index]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
kre = sys.argv[2] if len(sys.argv) > 2 else None
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"]
if kre:
    cmd += ["-k", "regex:" + kre]
rows = list(csv.reader(io.StringIO(subprocess.run(cmd, capture_output=True, text=True).stdout)))
blocks, cur = [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = {"name": r[1], "rows": []}
        blocks.append(cur)
    elif cur is not None:
        cur["rows"].append(r)
which = int(sys.argv[4]) if len(sys.argv) > 4 else 0
blk = blocks[which]
print(blk["name"], f"({len(blocks)} kernels in report)")
h = blk["rows"][0]
data = [r for r in blk["rows"][1:] if len(r) == len(h)]
ia, isrc, ie = h.index("Address"), h.index("Source"), h.index("Instructions Executed")
iss = h.index("Warp Stall Sampling (All Samples)")
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
ix = [h.index(c) for c in cols]
tot = sum(float(r[iss] or 0) for r in data)
agg = {c: sum(float(r[i] or 0) for r in data) for c, i in zip(cols, ix)}
T = sum(agg.values()) or 1
print("samples", tot, "warp instr", sum(float(r[ie] or 0) for r in data))
print("stalls:", {c[6:]: round(v / T * 100, 1) for c, v in sorted(agg.items(), key=lambda x: -x[1])[:8]})
base = int(data[0][ia], 16)
for r in sorted(data, key=lambda r: -float(r[iss] or 0))[:top]:
    v = {c[6:]: int(float(r[i] or 0)) for c, i in zip(cols, ix) if float(r[i] or 0) >= 2}
    print(f"{int(r[ia], 16) - base:6x} {float(r[iss]) / tot * 100:5.1f}% exec={r[ie]:>7} {r[isrc][:60]:60s} {v}")
