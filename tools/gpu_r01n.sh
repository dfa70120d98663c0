cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_r01n.log 2>&1; tail -3 gpurun_out/pytest_r01n.log; grep -E "^E  .*Error|^FAILED" gpurun_out/pytest_r01n.log | head
bash tools/gpu_ab.sh 3 simt build/ab/libad_p1.so build/ab/libad_v3.so build/ab/libad_v3.so::::AD_MAXREG=80
bash tools/gpu_ab.sh 2 simt build/ab/libad_p1.so build/ab/libad_v3.so
