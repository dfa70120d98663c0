cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
   -o gpurun_out/prof_simt_r01m python tools/prof_ls.py 2 simt 2 > gpurun_out/ncu_simt_r01m.log 2>&1; tail -1 gpurun_out/ncu_simt_r01m.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
   -o gpurun_out/prof_simt3_r01m python tools/prof_ls.py 3 simt 2 > gpurun_out/ncu_simt3_r01m.log 2>&1; tail -1 gpurun_out/ncu_simt3_r01m.log
timeout 900 python tools/accuracy_study.py gpurun_out/accuracy_r01.json > gpurun_out/accuracy_r01.log 2>&1; tail -3 gpurun_out/accuracy_r01.log
timeout 900 python bench.py > gpurun_out/bench_r01m.json 2> gpurun_out/bench_r01m.err; python -c "import json;d=json.load(open('gpurun_out/bench_r01m.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'])"
timeout 900 python bench.py --config 3 --steps 3 --no-cpu-baseline > gpurun_out/bench_r01m_cfg3.json 2>> gpurun_out/bench_r01m.err; python -c "import json;d=json.load(open('gpurun_out/bench_r01m_cfg3.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'])"
