cd $GRAFT_REPO_ROOT
bash tools/gpu_round.sh r01d tests
AD_DEBUG_LAUNCH=1 timeout 300 python tools/prof_ls.py 2 simt 1 2>&1 | grep libad | head -10
for eng in simt tc; do
  timeout 600 python bench.py --steps 10 --warmup 3 --engine $eng --no-cpu-baseline --no-paper-engine > gpurun_out/bench_r01d_$eng.json 2>>gpurun_out/bench_r01d.err
  python -c "import json;d=json.load(open('gpurun_out/bench_r01d_$eng.json'));print('$eng', '%.4g'%d['value'], d['config']['launch'])"
  for w in 3 4; do
    timeout 600 python bench.py --steps 10 --warmup 3 --engine $eng --warps $w --no-cpu-baseline --no-paper-engine > gpurun_out/bench_r01d_${eng}_w$w.json 2>>gpurun_out/bench_r01d.err
    python -c "import json;d=json.load(open('gpurun_out/bench_r01d_${eng}_w$w.json'));print('$eng w$w', '%.4g'%d['value'], d['config']['launch'])"
  done
done
tail -3 gpurun_out/bench_r01d.err
