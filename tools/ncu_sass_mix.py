"""Instruction mix of one kernel from an ncu report's SASS source page: executed warp-level
instructions per opcode class, and the hottest SASS lines by warp stall samples.

    python tools/ncu_sass_mix.py report.ncu-rep KERNEL_REGEX [top]
"""
import collections
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", "regex:" + kern], capture_output=True, text=True).stdout
lines = [l for l in out.splitlines() if l.strip()]
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"') or l.startswith("Address")
             or '"Source"' in l)
rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
hdr = rows[0]
print("columns:", hdr[:12], file=sys.stderr)
def col(*names):
    for n in names:
        for i, h in enumerate(hdr):
            if h.startswith(n):
                return i
    return None
isrc = col("Source")
iexe = col("Warp Instructions Executed", "Instructions Executed")
istall = col("Warp Stall Sampling (All Samples)", "Warp Stall Sampling")
mix = collections.Counter()
hot = []
tot = 0
for r in rows[1:]:
    if len(r) <= max(isrc, iexe):
        continue
    src = r[isrc].strip()
    try:
        n = float(r[iexe].replace(",", "")) if r[iexe] else 0.0
    except ValueError:
        continue
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    mix[op.split(".")[0]] += n
    tot += n
    if istall is not None:
        try:
            hot.append((float(r[istall].replace(",", "") or 0), src))
        except ValueError:
            pass
print(f"total warp instructions {tot:.4g}")
for op, n in mix.most_common(30):
    print(f"  {op:10s} {n:12.4g}  {100 * n / tot:5.1f}%")
if hot:
    print("hottest lines (stall samples):")
    for s, src in sorted(hot, reverse=True)[:top]:
        print(f"  {s:8.0f}  {src}")
