import sys, os, numpy as np, torch
sys.path.insert(0, os.environ.get('GRAFT_REPO_ROOT', '/root/repo'))
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth
w = synth.make_config(2)
ctx = ad.Context(0); ctx.upload_grid(w.grid); lid = ctx.upload_ligand(w.ligands[0], w.ff)
def run(phases, engine):
    g = torch.from_numpy(w.genes[:300].copy()).cuda()
    o = ctx.local_search(lid, g, max_iters=20, engine=engine, phases=phases)
    torch.cuda.synchronize()
    return o["best_energy"].cpu().numpy(), g.cpu().numpy()
for eng in ("simt", "tc"):
    a = run(False, eng); b = run(False, eng); c = run(True, eng)
    d = np.abs(a[0].astype(np.float64) - c[0]) / (1 + np.abs(a[0]))
    print(os.environ.get("AD_NO_CH"), eng, "plain-plain equal:", np.array_equal(a[0], b[0]), "plain-instr equal:", np.array_equal(a[0], c[0]), "max rel diff %.3g" % d.max(), "n diff", int((a[0] != c[0]).sum()))
np.savez(f"/tmp/det_{os.environ.get('AD_NO_CH', '0')}.npz", simt=run(False, "simt")[0], simt_i=run(True, "simt")[0])
if os.environ.get("AD_NO_CH"):
    x, y = np.load("/tmp/det_0.npz"), np.load("/tmp/det_1.npz")
    print("CH-plain == generic-plain:", np.array_equal(x["simt"], y["simt"]), " CH-instr == generic-plain:",
          np.array_equal(x["simt_i"], y["simt"]))
