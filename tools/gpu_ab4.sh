cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider 2>&1 | tail -3
timeout 1200 python tools/ab.py 2 simt build/ab/libad_cell.so:::xpair build/ab/libad_cell.so:::cell build/ab/libad_cell.so::hybrid:cell 2>&1 | tail -4
timeout 1200 python tools/ab.py 2 tc build/ab/libad_cell.so:::xpair build/ab/libad_cell.so:::cell 2>&1 | tail -3
