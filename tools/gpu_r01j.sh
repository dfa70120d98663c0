cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_r01j.log 2>&1; tail -3 gpurun_out/pytest_r01j.log; grep -E "^E  .*AssertionError|^FAILED" gpurun_out/pytest_r01j.log | head
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" 2>&1 | tail -2
timeout 1200 python tools/ab.py 2 simt build/ab/libad_h.so build/ab/libad_j.so 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_r01j.json 2> gpurun_out/bench_r01j.err; tail -c 3000 gpurun_out/bench_r01j.json
