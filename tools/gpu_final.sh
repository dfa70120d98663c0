#!/bin/bash
# Round-end measurement set on one B200: bash tools/gpu_final.sh TAG [screen|-] [ncu]
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-final}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_${TAG}_default.json 2> gpurun_out/bench_${TAG}_default.err
timeout 900 python bench.py --config 3 --steps 3 --warmup 3 > gpurun_out/bench_${TAG}_cfg3.json 2> gpurun_out/bench_${TAG}_cfg3.err
timeout 900 python bench.py --engine tc --no-cpu-baseline --no-paper-engine > gpurun_out/bench_${TAG}_tc.json 2> gpurun_out/bench_${TAG}_tc.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_${TAG}_ref.json 2> gpurun_out/bench_${TAG}_ref.err
[ "$2" = screen ] && timeout 1800 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/bench_${TAG}_cfg5.json 2> gpurun_out/bench_${TAG}_cfg5.err
timeout 900 python tools/phases.py gpurun_out/phases_${TAG}.json 2,3 > gpurun_out/phases_${TAG}.txt 2>&1
bash tools/gpu_round.sh $TAG launches
[ "$3" = ncu ] && bash tools/gpu_round.sh $TAG ncu ncu_simt && rm -f gpurun_out/prof_simt_$TAG.ncu-rep  # (the config-2 SIMT capture again under ncu_simt; gpurun_out <= 64 MiB)
python - <<PY
import json
for k in ("default", "cfg3", "tc", "ref", "cfg5"):
    try:
        d = json.load(open(f"gpurun_out/bench_${TAG}_{k}.json"))
    except Exception as e:
        print(k, "missing", e); continue
    print(k, d.get("value"), d.get("ms_per_step"), (d.get("roofline") or {}).get("frac"), d.get("clocks"))
PY
