cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
   -o gpurun_out/prof_simt_r01k python tools/prof_ls.py 2 simt 2 > gpurun_out/ncu_simt_r01k.log 2>&1; tail -2 gpurun_out/ncu_simt_r01k.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 \
   -o gpurun_out/prof_simt3_r01k python tools/prof_ls.py 3 simt 2 > gpurun_out/ncu_simt3_r01k.log 2>&1; tail -2 gpurun_out/ncu_simt3_r01k.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01k.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_r01k.log 2>&1; wc -l gpurun_out/launches_r01k.csv
