"""Summarise an `ncu --set full` report (one row per captured launch) into JSON.
Usage: python tools/ncu_summary.py report.ncu-rep > summary.json"""
import csv
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed": "tensor_pipe_active_pct",
    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed": "tensor_pipe_active_realtime_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "lts__t_sectors.avg.pct_of_peak_sustained_elapsed": "l2_sectors_pct",
    "lts__t_sectors.sum": "l2_sectors",
    "l1tex__data_bank_reads.avg.pct_of_peak_sustained_elapsed": "smem_bank_reads_pct",
    "l1tex__data_bank_writes.avg.pct_of_peak_sustained_elapsed": "smem_bank_writes_pct",
    "launch__registers_per_thread": "registers_per_thread",
    "launch__block_size": "block_size",
    "launch__grid_size": "grid_size",
    "sm__cycles_active.avg": "sm_cycles_active",
    "smsp__cycles_active.avg.pct_of_peak_sustained_elapsed": "smsp_active_pct",
    "sm__inst_executed.sum": "warp_instructions",
}

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, units = rows[0], rows[1]
res = []
for r in rows[2:]:
    d = {"kernel": r[hdr.index("Kernel Name")][:120]}
    for k, name in KEYS.items():
        if k in hdr:
            i = hdr.index(k)
            v = r[i].replace(",", "")
            try:
                v = float(v)
            except ValueError:
                pass
            d[name] = v
            d[name + "_unit"] = units[i]
    res.append(d)
print(json.dumps(res, indent=1))
