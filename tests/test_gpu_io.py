"""NEXT-4 on the GPU: ligands and receptor maps read from PDBQT / AutoGrid files
(paper_conf_sc_solis_vasquezts25_b200/io.py) go through the C ABI and meet the
same parity gates against the FP64 oracle as the generated arrays
(tests/parity.py), and the docking CLI (dock.py, the artifact
command of P:L520-521) runs end to end."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import io as adio  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402
from tests import parity as P  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def files(tmp_path_factory):
    d = tmp_path_factory.mktemp("autogrid")
    names = synth.TYPESETS[6]
    L = synth.make_config(2).ligands[0]
    g = synth.make_grid(2100, 61, names, 2000)
    adio.write_maps(g, names, str(d / "rec"))
    adio.write_pdbqt(L, str(d / "lig.pdbqt"), centroid=(0.2, -0.1, 0.3))
    return str(d / "rec.maps.fld"), str(d / "lig.pdbqt")


def test_file_inputs_meet_the_gates(files):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import ad
    fld, pdbqt = files
    G, names = adio.read_fld(fld)
    L, c = adio.read_pdbqt(pdbqt, names)
    ff = synth.FFParams()
    rng = np.random.default_rng(3)
    around = adio.input_genes(c, G, L.n_tors)[:3]
    from paper_conf_sc_solis_vasquezts25_b200.dock import random_starts
    genes = random_starts(rng, 256, L.n_tors, G, around)
    genes[0] = adio.input_genes(c, G, L.n_tors)
    ctx = ad.Context(0)
    try:
        ctx.upload_grid(G)
        lid = ctx.upload_ligand(L, ff)
        gd = torch.from_numpy(genes).cuda()
        ctx.local_search(lid, gd, max_iters=100, engine="simt")
        torch.cuda.synchronize()
        relaxed = gd.cpu().numpy()
        for gs in (genes, relaxed):
            E, Gr, _ = ctx.score(lid, torch.from_numpy(gs).cuda(), grad=True)
            torch.cuda.synchronize()
            Eo, Go, aux, ag = O.score(L, G, ff, gs)
            Gn = L.n_genes
            kink = aux[:, O.AUX_MARGIN_G] < 1e-4
            assert np.all(P.energy_gate(E.cpu().numpy(), Eo, aux))
            assert np.all(P.grad_gate(Gr.cpu().numpy()[:, :Gn], Go[:, :Gn], ag[:, :Gn]) | kink)
    finally:
        ctx.close()


def test_dock_cli_runs(files, tmp_path):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import dock
    fld, pdbqt = files
    out = tmp_path / "res.json"
    runs = dock.main(["--ffile", fld, "--lfile", pdbqt, "--nrun", "4", "--pop", "32", "--lsit", "50",
                      "--out", str(out)])
    assert len(runs) == 4 and all(np.isfinite(r["energy"]) for r in runs) and out.exists()
    runs_lga = dock.main(["--ffile", fld, "--lfile", pdbqt, "--nrun", "2", "--pop", "16", "--lsit", "10",
                          "--lga", "--ngen", "3", "--nev", "100000000"])
    assert len(runs_lga) == 2 and all(np.isfinite(r["energy"]) for r in runs_lga)
