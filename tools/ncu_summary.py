"""Summarise an ncu --set full report: key SOL / occupancy / stall / shared-memory metrics."""
import csv
import io
import re
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__block_size", "launch__grid_size", "launch__occupancy_limit_registers",
    "launch__occupancy_limit_shared_mem", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__inst_executed.sum", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "lts__t_bytes.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard", 
]
STALL = re.compile(r"smsp__pcsamp_warps_issue_stalled_([a-z_]+)$")


def summary(path):
    out = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    d = {k: (val, unit) for k, unit, val in zip(h, u, v)}
    res = {}
    for k in KEYS:
        if k in d:
            res[k] = d[k]
    stalls = {}
    for k, (val, unit) in d.items():
        m = STALL.search(k)
        if m and not m.group(1).endswith("not_issued"):
            try:
                stalls[m.group(1)] = float(val.replace(",", ""))
            except ValueError:
                pass
    tot = sum(stalls.values()) or 1
    res["stalls_pct"] = {k: round(100 * v / tot, 1) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1]) if v / tot > 0.01}
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(p)
        for k, v in summary(p).items():
            print(f"  {k:70s} {v}")
