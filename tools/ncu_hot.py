"""Top SASS instructions of one kernel by a stall column (ncu source page): where a stall reason
comes from.  usage: ncu_hot.py REP KERNEL_REGEX [stall_col] [n]"""
import csv, subprocess, sys
rep, kre = sys.argv[1], sys.argv[2]
col = sys.argv[3] if len(sys.argv) > 3 else "stall_long_sb"
n = int(sys.argv[4]) if len(sys.argv) > 4 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", "regex:" + kre], capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out[1:]))
hdr = rows[0]
body = []
for r in rows[1:]:  # the first launch's section only (later launches repeat the listing)
    if r and r[0] == "Kernel Name":
        break
    if len(r) == len(hdr):
        body.append(r)
ci, si, ai = hdr.index(col), hdr.index("Source"), hdr.index("Address")
tot = sum(float(r[ci] or 0) for r in body) or 1.0
allc = hdr.index("Warp Stall Sampling (All Samples)")
print(f"{col}: {tot:.0f} samples of {sum(float(r[allc] or 0) for r in body):.0f}")
idx = {r[ai]: i for i, r in enumerate(body)}
for r in sorted(body, key=lambda r: -float(r[ci] or 0))[:n]:
    i = idx[r[ai]]
    print(f"{100*float(r[ci])/tot:5.1f}%  {i:5d}  {r[si].strip()[:90]}")
