cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_r02i_default.json 2> gpurun_out/bench_r02i_default.err
timeout 900 python bench.py --config 3 --steps 3 --warmup 3 > gpurun_out/bench_r02i_cfg3.json 2> gpurun_out/bench_r02i_cfg3.err
timeout 900 python tools/phases.py gpurun_out/phases_r02i.json 2,3 > gpurun_out/phases_r02i.txt 2>&1
bash tools/gpu_round.sh r02i ncu_simt launches
python -c "import json;d=json.load(open('gpurun_out/bench_r02i_default.json'));print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['config1_score_call'], (d['parity'] or {}).get('relaxed_poses'))"
