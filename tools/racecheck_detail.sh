cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/rc
CASES="score_c1_grad score_c2_grad ls_c2_simt ls_c2_tc ls_c2_tc_fp16 ls_c2_paper ls_c2_paper_tcec ls_c3_simt ls_c3_tc ls_c3_paper screen lga reduce ls_c2_simt:AD_PK_SMEM_MAX=0 ls_c2_simt:AD_PK_SMEM_MAX=0,AD_PAIRS_SMEM_MAX=0 ls_c2_simt:AD_INTRA_MODE=owner ls_c2_simt:AD_INTRA_MODE=hybrid"
for c in $CASES; do
  timeout 600 compute-sanitizer --print-limit 0 --tool racecheck --racecheck-report all python tools/sanitize_cases.py $c 2>&1 | python tools/racecheck_summary.py > gpurun_out/rc/$c.txt
  head -3 gpurun_out/rc/$c.txt
done
