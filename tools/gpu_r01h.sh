cd $GRAFT_REPO_ROOT
timeout 300 ncu --metrics l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum --csv --log-file gpurun_out/bank_probe.csv build/bank_probe > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_screen.py -q -x -p no:cacheprovider > gpurun_out/screen_test.log 2>&1; tail -30 gpurun_out/screen_test.log | grep -E "Error|assert|passed|failed" | head
timeout 1200 python tools/ab.py 2 simt build/ab/libad_cell.so build/ab/libad_h.so 2>&1 | tail -3
timeout 1200 python tools/ab.py 3 simt build/ab/libad_h.so 2>&1 | tail -2
