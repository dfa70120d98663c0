cd $GRAFT_REPO_ROOT
bash tools/gpu_round.sh r01e tests smoke
for eng in simt tc; do
  timeout 900 python bench.py --steps 10 --warmup 3 --engine $eng $( [ $eng = tc ] && echo --no-cpu-baseline ) > gpurun_out/bench_r01e_$eng.json 2>> gpurun_out/bench_r01e.err
  python -c "import json;d=json.load(open('gpurun_out/bench_r01e_$eng.json'));print('$eng', '%.4g'%d['value'], 'frac %.3f'%d['roofline']['frac'], d['config']['launch'], d['clocks'], d['paper_baseline_engine'], d['parity'], d['cpu_baseline'], d['e2e'])"
done
timeout 900 python bench.py --steps 3 --warmup 3 --config 3 --no-cpu-baseline > gpurun_out/bench_r01e_cfg3.json 2>> gpurun_out/bench_r01e.err
python -c "import json;d=json.load(open('gpurun_out/bench_r01e_cfg3.json'));print('cfg3', '%.4g'%d['value'], 'frac %.3f'%d['roofline']['frac'], d['config']['launch'], d['paper_baseline_engine'])"
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_r01e_ref.json 2>> gpurun_out/bench_r01e.err; cat gpurun_out/bench_r01e_ref.json | head -c 600
bash tools/gpu_round.sh r01e ncu launches
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_block_baseline -s 1 -c 1 -o gpurun_out/prof_paper_r01e python tools/prof_ls.py 2 paper 2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_block_baseline -s 1 -c 1 -o gpurun_out/prof_papertcec_r01e python tools/prof_ls.py 2 paper_tcec 2 > /dev/null 2>&1
tail -3 gpurun_out/bench_r01e.err
