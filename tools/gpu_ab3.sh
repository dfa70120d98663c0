cd $GRAFT_REPO_ROOT
timeout 1200 python tools/ab.py 2 simt build/ab/libad_m64.so build/ab/libad_m72.so build/ab/libad_m80.so build/ab/libad_m72.so::hybrid build/ab/libad_m64.so::hybrid 2>&1 | tail -6
timeout 1200 python tools/ab.py 3 simt build/ab/libad_m64.so build/ab/libad_m72.so build/ab/libad_m80.so 2>&1 | tail -4
