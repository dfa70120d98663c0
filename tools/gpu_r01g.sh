cd $GRAFT_REPO_ROOT
timeout 300 ncu --metrics l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum --csv build/bank_probe 2>/dev/null | grep -E "probe|wavefronts|conflicts" | awk -F'","' '{print $5, $(NF-2), $NF}' | head -30
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -3
timeout 1200 python tools/ab.py 2 simt build/ab/libad_cell.so build/ab/libad_g.so 2>&1 | tail -3
timeout 1200 python tools/ab.py 3 simt build/ab/libad_cell.so build/ab/libad_g.so build/ab/libad_g.so:16 2>&1 | tail -4
