#!/bin/bash
# Config 5 (virtual screen) on the GPU box: test, a small run, full runs per schedule effort.
#   bash tools/gpu_screen.sh TAG [efforts...]
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-dev}; shift
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_screen.py -q -p no:cacheprovider > gpurun_out/pytest_screen_$TAG.log 2>&1; tail -1 gpurun_out/pytest_screen_$TAG.log
timeout 600 python bench.py --config 5 --ligands 512 --steps 2 --warmup 1 > gpurun_out/bench5_small_$TAG.json 2> gpurun_out/bench5_small_$TAG.err
tail -2 gpurun_out/bench5_small_$TAG.err; cut -c1-400 gpurun_out/bench5_small_$TAG.json
for e in "$@"; do
  timeout 1200 python bench.py --config 5 --steps 3 --warmup 3 --effort $e > gpurun_out/bench5_e${e}_$TAG.json 2> gpurun_out/bench5_e${e}_$TAG.err
  tail -2 gpurun_out/bench5_e${e}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench5_e${e}_$TAG.json'));print('effort $e', '%.4g'%d['value'], 'e2e %.4g'%d['e2e']['value'], 'frac %.3f'%d['roofline']['frac'], d['config']['setup_s_rank0'], d['parity'], d['cpu_baseline'])"
done
