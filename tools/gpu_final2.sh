#!/bin/bash
# Round-end evidence set on one B200: bash tools/gpu_final2.sh TAG
#   tests + smoke, default bench, config 3, TC engine, --impl reference, A14 phases,
#   launch list, ncu --set full of the config-2 / config-3 SIMT LS kernels (text summaries)
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-final}
mkdir -p gpurun_out
bash tools/gpu_round.sh $TAG tests smoke > /dev/null 2>&1
tail -2 gpurun_out/pytest_gpu_$TAG.log; tail -1 gpurun_out/smoke_$TAG.log
bash tools/gpu_final.sh $TAG - > gpurun_out/final_$TAG.txt 2>&1; tail -6 gpurun_out/final_$TAG.txt
bash tools/gpu_round.sh $TAG ncu_simt > /dev/null 2>&1
for c in 2 3; do
  python tools/ncu_summary.py gpurun_out/prof_simt_c${c}_$TAG.ncu-rep > gpurun_out/ncu_summary_c${c}_$TAG.txt 2>&1
  ncu -i gpurun_out/prof_simt_c${c}_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/sass_c${c}_$TAG.csv 2>/dev/null
  rm -f gpurun_out/prof_simt_c${c}_$TAG.ncu-rep
done
ls gpurun_out | wc -l
