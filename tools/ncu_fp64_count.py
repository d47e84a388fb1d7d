"""Count executed fp64 pipe thread-instructions (DADD/DMUL/DFMA, predicated on) per kernel from
an ncu report's SASS source page: python tools/ncu_fp64_count.py report.ncu-rep kernel_regex"""
import collections
import csv
import subprocess
import sys

rep, kname = sys.argv[1], sys.argv[2]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", "regex:" + kname, "-c", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
i_src = hdr.index("Source")
i_t = hdr.index("Predicated-On Thread Instructions Executed")
i_w = hdr.index("Instructions Executed")
cnt = collections.Counter()
tot_w = 0.0
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    toks = r[i_src].split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith("@") else toks[0]
    op = op.split(".")[0]
    try:
        cnt[op] += float(r[i_t])
        tot_w += float(r[i_w])
    except ValueError:
        pass
fp64 = cnt["DADD"] + cnt["DMUL"] + cnt["DFMA"]
print(f"fp64_thread_inst {fp64:.0f} (DADD {cnt['DADD']:.0f} DMUL {cnt['DMUL']:.0f} "
      f"DFMA {cnt['DFMA']:.0f}); all warp inst {tot_w:.0f}; MUFU {cnt['MUFU']:.0f}; "
      f"DSETP {cnt['DSETP']:.0f}")
