cd $GRAFT_REPO_ROOT
rm -f gpurun_out/sched.bin
AD_DUMP_SCHEDULE=gpurun_out/sched.bin timeout 300 python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth
for c in (2,3):
    w=synth.make_config(c); ctx=ad.Context(0); ctx.upload_grid(w.grid); ctx.upload_ligand(w.ligands[0], w.ff); ctx.close()
print('ok')
"
ls -la gpurun_out/sched.bin
