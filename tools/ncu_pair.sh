cd $GRAFT_REPO_ROOT
for v in vC2 vC5; do
  AD_LIB=$PWD/ab/$v.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_warp_engine -s 1 -c 1 -o gpurun_out/prof_c3_$v python tools/prof_ls.py 3 simt 2 > gpurun_out/ncu_c3_$v.log 2>&1
done
ls -la gpurun_out
