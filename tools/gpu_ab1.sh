cd $GRAFT_REPO_ROOT
timeout 1200 python tools/ab.py 2 simt build/ab/libad_r96_c8.so build/ab/libad_r96_c8.so:3 build/ab/libad_r80_c8.so build/ab/libad_r80_c1.so build/ab/libad_r88_c4.so 2>&1 | tail -8
timeout 600 python tools/ab.py 2 tc build/ab/libad_r96_c8.so build/ab/libad_r80_c1.so 2>&1 | tail -3
