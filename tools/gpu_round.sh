#!/bin/bash
# One GPU iteration: tests, bench lines, optional ncu captures.
#   bash tools/gpu_round.sh TAG [tests] [smoke] [bench] [bench1] [bench3] [ncu] [ncu_simt] [sanitize] [ncu_paper] [accuracy] [reduce] [ab] [launches]
#   (ab: AB_LIBS='lib1.so lib2.so ...' in the environment)
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-dev}; shift
mkdir -p gpurun_out
for what in "$@"; do
  case $what in
    tests)
      timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
      echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log; tail -4 gpurun_out/pytest_gpu_$TAG.log ;;
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -2 gpurun_out/smoke_$TAG.log ;;
    bench1)
      timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-paper-engine > gpurun_out/bench_${TAG}_simt.json 2>> gpurun_out/bench_$TAG.err
      python -c "import json;d=json.load(open('gpurun_out/bench_${TAG}_simt.json'));print('simt', '%.4g'%d['value'], d['ms_per_step'], 'frac %.3f'%d['roofline']['frac'], d['clocks'])" ;;
    bench)
      for eng in tc simt; do
        timeout 900 python bench.py --steps 10 --warmup 3 --engine $eng $( [ $eng = simt ] && echo --no-cpu-baseline ) \
          > gpurun_out/bench_${TAG}_$eng.json 2>> gpurun_out/bench_$TAG.err
        python -c "import json;d=json.load(open('gpurun_out/bench_${TAG}_$eng.json'));print('$eng', '%.4g'%d['value'], 'frac %.3f'%d['roofline']['frac'], d['clocks'], (d.get('paper_baseline_engine') or {}).get('speedup_of_this_engine'))"
      done ;;
    bench3)
      timeout 900 python bench.py --steps 3 --warmup 3 --config 3 --engine simt --no-cpu-baseline --no-paper-engine > gpurun_out/bench_${TAG}_cfg3.json 2>> gpurun_out/bench_$TAG.err
      python -c "import json;d=json.load(open('gpurun_out/bench_${TAG}_cfg3.json'));print('cfg3', '%.4g'%d['value'], 'frac %.3f'%d['roofline']['frac'], (d.get('paper_baseline_engine') or {}).get('speedup_of_this_engine'))" ;;
    ncu)
      for eng in tc simt; do
        timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
          -o gpurun_out/prof_${eng}_$TAG python tools/prof_ls.py 2 $eng 2 > gpurun_out/ncu_${eng}_$TAG.log 2>&1
      done ;;
    ncu_simt)
      for cfg in 2 3; do
        timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
          -o gpurun_out/prof_simt_c${cfg}_$TAG python tools/prof_ls.py $cfg simt 2 > gpurun_out/ncu_simt_c${cfg}_$TAG.log 2>&1
      done ;;
    sanitize)
      bash tools/sanitize.sh $TAG ;;
    ncu_paper)
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_block_baseline -s 1 -c 1 \
        -o gpurun_out/prof_paper_$TAG python tools/prof_ls.py 2 paper 2 > gpurun_out/ncu_paper_$TAG.log 2>&1 ;;
    accuracy)
      AD_STUDY_OUT=gpurun_out/accuracy_$TAG.json timeout 900 python -m pytest tests/test_gpu_accuracy_study.py -m gpu -q -s -p no:cacheprovider > gpurun_out/accuracy_$TAG.log 2>&1; tail -3 gpurun_out/accuracy_$TAG.log ;;
    reduce)
      timeout 900 python tools/bench_reduce.py gpurun_out/reduce_$TAG.json 100 > gpurun_out/reduce_$TAG.log 2>&1; tail -25 gpurun_out/reduce_$TAG.log ;;
    ab)
      timeout 1200 python tools/ab.py 2 simt $AB_LIBS 2>&1 | tail -8 ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
        python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-paper-engine > gpurun_out/bench_under_ncu_$TAG.log 2>&1 ;;
  esac
done
ls gpurun_out | tail -30
