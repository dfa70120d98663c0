cd $GRAFT_REPO_ROOT
bash tools/gpu_ab.sh 2 simt build/ab/libad_v3.so build/ab/libad_rg.so
bash tools/gpu_ab.sh 3 simt build/ab/libad_v3.so build/ab/libad_rg.so build/ab/libad_rg.so::::AD_MAXREG=80
