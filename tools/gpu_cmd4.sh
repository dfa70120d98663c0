cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 -o gpurun_out/prof_tc_r01 python tools/prof_ls.py 2 tc 2 > gpurun_out/ncu_tc.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 -o gpurun_out/prof_simt_r01 python tools/prof_ls.py 2 simt 2 > gpurun_out/ncu_simt.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_block_baseline -s 1 -c 1 -o gpurun_out/prof_paper_r01 python tools/prof_ls.py 2 paper 2 > gpurun_out/ncu_paper.log 2>&1
ls -la gpurun_out; tail -2 gpurun_out/ncu_tc.log
