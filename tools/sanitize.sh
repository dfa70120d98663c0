#!/bin/bash
# compute-sanitizer gate over every kernel family (tools/sanitize_cases.py):
#   bash tools/sanitize.sh TAG [tools...]    (default: racecheck synccheck memcheck initcheck)
# One process per tool runs every case (the sanitizer report names the kernel and
# the "=== case" lines in the log name the case); AD_PKG is read once per process,
# so the config-3 scatter-gmem case runs in a second process.  Logs under
# gpurun_out/sanitize_TAG/, one summary line per process in summary.txt.
# Pair-loop modes through libad's A/B knobs: cherry (default, small ligands),
# scatter-smem (AD_PK_SMEM_MAX=0), scatter-gmem (+ AD_PAIRS_SMEM_MAX=0), packed-gmem
# (config 3 default), scatter-gmem on config 3 (AD_PKG=0), owner / hybrid (AD_INTRA_MODE).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-dev}; shift
TOOLS=${*:-racecheck synccheck memcheck initcheck}
OUT=gpurun_out/sanitize_$TAG
mkdir -p $OUT
CASES="score_c1_grad score_c1_energy score_c2_grad ls_c1_simt ls_c2_simt ls_c2_tc ls_c2_tc_fp16 ls_c2_paper
 ls_c2_paper_tcec ls_c3_simt ls_c3_tc ls_c3_paper screen lga reduce
 ls_c2_simt:AD_PK_SMEM_MAX=0 ls_c2_simt:AD_PK_SMEM_MAX=0,AD_PAIRS_SMEM_MAX=0
 ls_c2_simt:AD_INTRA_MODE=owner ls_c2_simt:AD_INTRA_MODE=hybrid ls_c2_tc:AD_INTRA_MODE=owner
 ls_c3_simt:AD_GRID_LAYOUT=cell ls_c2_simt:AD_GRID_LAYOUT=xpair"
for tool in $TOOLS; do
  extra=""
  [ $tool = racecheck ] && extra="--racecheck-report all"
  [ $tool = memcheck ] && extra="--leak-check no"
  for part in main pkg0; do
    if [ $part = main ]; then cs=$CASES; envs=""; else cs="ls_c3_simt ls_c3_tc"; envs="AD_PKG=0"; fi
    env $envs timeout 2400 compute-sanitizer --error-exitcode 9 --print-limit 50 --tool $tool $extra \
      python tools/sanitize_cases.py $cs > $OUT/${tool}_$part.log 2>&1
    rc=$?
    ok=$(grep -c "^case ok" $OUT/${tool}_$part.log)
    summ=$(grep -E "ERROR SUMMARY|RACECHECK SUMMARY" $OUT/${tool}_$part.log | tail -1)
    echo "$tool $part $envs rc=$rc cases_ok=$ok ${summ:-no summary}" | tee -a $OUT/summary.txt
  done
done
