cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_r01i.log 2>&1; tail -3 gpurun_out/pytest_r01i.log; grep -E "^E  .*AssertionError|^FAILED" gpurun_out/pytest_r01i.log | head
timeout 1200 python tools/ab.py 2 simt build/ab/libad_h.so build/ab/libad_i.so 2>&1 | tail -3
timeout 1200 python tools/ab.py 3 simt build/ab/libad_h.so build/ab/libad_i.so 2>&1 | tail -3
