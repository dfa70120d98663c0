#!/bin/bash
# Per-library ncu counters of one config-2 LS launch (instructions, shared wavefronts,
# issue activity, duration): bash tools/gpu_counters.sh TAG LIB...
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=$1; shift
M=smsp__inst_executed.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,l1tex__throughput.avg.pct_of_peak_sustained_active,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum
for lib in "$@"; do
  AD_LIB=$(realpath $lib) timeout 600 ncu --metrics $M --clock-control none -k regex:k_warp_engine -s 1 -c 1 --csv \
    python tools/prof_ls.py 2 simt 2 2>/dev/null | grep -E '"(smsp|l1tex|gpu)__' | awk -F'","' -v L=$(basename $lib) '{print L, $(NF-2), $NF}' | tr -d '"'
done | tee gpurun_out/counters_$TAG.txt
