cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_r01l.log 2>&1; tail -3 gpurun_out/pytest_r01l.log; grep -E "^E  .*Error|^FAILED" gpurun_out/pytest_r01l.log | head
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" 2>&1 | tail -1
bash tools/gpu_ab.sh 2 simt build/ab/libad_rb2.so build/ab/libad_z.so
timeout 900 python tools/accuracy_study.py gpurun_out/accuracy_r01.json > gpurun_out/accuracy_r01.log 2>&1; tail -5 gpurun_out/accuracy_r01.log
