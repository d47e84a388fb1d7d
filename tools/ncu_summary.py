"""Summarise an ncu --set full report into per-kernel counters used by bench.py's roofline:
DRAM bytes and executed fp64 (DADD/DMUL/DFMA) thread instructions per launch, per owned zone.

    python tools/ncu_summary.py report.ncu-rep ZONES [KERNEL=ZONES ...] > profiles/kernel_counters.json

ZONES: owned zones one launch covers; KERNEL=ZONES overrides it per kernel key (e.g. the grouped
zone stage covers every domain of the GPU, a node-stage launch one domain).
"""
import csv
import json
import subprocess
import sys

rep, zones_all = sys.argv[1], float(sys.argv[2])
zones_of = {kv.split("=")[0]: float(kv.split("=")[1]) for kv in sys.argv[3:]}
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout.splitlines()
rows = list(csv.reader(raw))
hdr = rows[0]
out = {}
for vals in rows[2:]:
    d = dict(zip(hdr, vals))
    name = d["Kernel Name"]
    key = "k_zone_stage" if "k_zone_stage" in name else (
        "k_cycle_fused" if "k_cycle<" in name and ", 1>" in name else (
            "k_node_energy" if "k_cycle<" in name else name.split("(")[0]))
    if key in out:
        continue
    zones = zones_of.get(key, zones_all)
    def f(k):
        try:
            return float(d[k].replace(",", ""))
        except (KeyError, ValueError):
            return float("nan")
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1.0, "KB": 1e3,
             "MB": 1e6, "GB": 1e9}
    units = dict(zip(hdr, rows[1]))
    rd = f("dram__bytes_read.sum") * scale[units["dram__bytes_read.sum"]]
    wr = f("dram__bytes_write.sum") * scale[units["dram__bytes_write.sum"]]
    unit = 1.0  # bytes (ncu scales each metric's unit; the units row says which)
    regex = "k_zone_stage" if key == "k_zone_stage" else "k_cycle"
    fp = subprocess.run([sys.executable, "tools/ncu_fp64_count.py", rep, regex],
                        capture_output=True, text=True).stdout.split()
    fp64 = float(fp[1]) if len(fp) > 1 else float("nan")
    out[key] = {
        "duration_us": f("gpu__time_duration.sum") * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0,
                                                      "us": 1.0, "msecond": 1e3, "ms": 1e3}[units["gpu__time_duration.sum"]],
        "dram_bytes": (rd + wr) * unit, "dram_read_bytes": rd * unit, "dram_write_bytes": wr * unit,
        "zones_per_launch": zones,
        "dram_bytes_per_zone": (rd + wr) * unit / zones,
        "fp64_inst": fp64, "fp64_inst_per_zone": fp64 / zones,
        "fp64_pipe_pct": f("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
        "issue_active": f("smsp__issue_active.avg.per_cycle_active"),
        "warps_active": f("sm__warps_active.avg.per_cycle_active"),
        "registers": f("launch__registers_per_thread"),
        "warp_inst": f("smsp__inst_executed.sum"),
        # shared-memory data-pipe wavefronts (the node stage's binding resource)
        "smem_wavefronts": f("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
        "smem_wavefronts_pct": f("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"
                                 ".pct_of_peak_sustained_elapsed"),
    }
json.dump({"report": rep, "zones": zones_all, "kernels": out}, sys.stdout, indent=1)
print()
