cd $GRAFT_REPO_ROOT
bash tools/gpu_round.sh own tests
for mode in scatter owner; do
  for eng in tc simt; do
    AD_INTRA_MODE=$mode timeout 600 python bench.py --steps 10 --warmup 3 --engine $eng --no-cpu-baseline --no-paper-engine > gpurun_out/bench_mode_${mode}_$eng.json 2>>gpurun_out/bench_modes.err
    python -c "import json;d=json.load(open('gpurun_out/bench_mode_${mode}_$eng.json'));print('$mode $eng', '%.4g'%d['value'], d['config']['launch'])"
  done
  AD_INTRA_MODE=$mode timeout 600 python bench.py --steps 2 --warmup 2 --config 3 --engine simt --no-cpu-baseline --no-paper-engine > gpurun_out/bench_mode_${mode}_cfg3.json 2>>gpurun_out/bench_modes.err
  python -c "import json;d=json.load(open('gpurun_out/bench_mode_${mode}_cfg3.json'));print('$mode cfg3', '%.4g'%d['value'], d['config']['launch'])"
done
AD_INTRA_MODE=owner timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 -o gpurun_out/prof_simt_own python tools/prof_ls.py 2 simt 2 > /dev/null 2>&1
tail -3 gpurun_out/bench_modes.err
