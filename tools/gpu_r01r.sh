cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_r01r.log 2>&1; tail -2 gpurun_out/pytest_r01r.log; grep -E "^FAILED" gpurun_out/pytest_r01r.log | head
bash tools/gpu_ab.sh 3 simt build/ab/libad_cq2.so build/ab/libad_sp2.so
bash tools/gpu_ab.sh 2 simt build/ab/libad_cq2.so build/ab/libad_sp2.so
