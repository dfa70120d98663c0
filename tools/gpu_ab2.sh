cd $GRAFT_REPO_ROOT
AD_INTRA_MODE=hybrid timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "score_poses or shadowed or full_size" 2>&1 | tail -3
timeout 1200 python tools/ab.py 2 simt build/ab/libad_cur.so::scatter build/ab/libad_cur.so::hybrid build/ab/libad_cur80.so::scatter build/ab/libad_cur80.so::hybrid 2>&1 | tail -5
timeout 1200 python tools/ab.py 3 simt build/ab/libad_cur.so::scatter build/ab/libad_cur.so::hybrid 2>&1 | tail -3
