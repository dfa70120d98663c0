"""Seeded synthetic inputs shaped like the paper's docking workloads.

This module is the ONLY code shared by the CUDA path and the FP64 oracle
(`oracle/`).  It draws random ligands, receptor grid maps and start genotypes;
it contains none of the method's arithmetic (no pose building, no grid
interpolation, no pair energies, no reductions, no ADADELTA).  Everything it
returns is a plain array that both sides consume as input.

Workload shapes follow BASELINE.json `configs` and SURVEY.md §8(d):

  config 1  tiny      12 atoms,  2 torsions, 3 types, 32^3 grid,  256 poses
  config 2  drug-like 40 atoms,  8 torsions, 6 types, 60^3 grid,  20 runs x 150 pop
  config 3  large     110 atoms, 32 torsions, 8 types, 96^3 grid, 100 runs x 150 pop
  config 4  reduction microbench partials (C x P per block)
  config 5  screen    8192 ligands, N ~ U{20..110}, T ~ U{0..min(32, N//3)}, 20 runs x 16 pop

Seeds: seed = 1000 * config + replica.

Ligand recipe (readings Z9/Z13/Z22 in DESIGN.md):
  * a random tree, bonds 1.5 +- 0.05 A, bond angles 109.5 +- 5 deg, no two atoms
    closer than 2.3 A except bonded ones (>= 2.9 A beyond 1-3 neighbours);
  * rotatable bonds are T randomly chosen non-terminal tree edges; rigid
    fragments are the components left after cutting them; the root fragment
    is the most central fragment of the torsion tree;
  * tors_axis[b] = (a, c): a on the root side, c on the moving side;
    tors_moving[b] = atoms on c's side; torsions are listed root -> leaf;
  * pair list: atoms in different rigid fragments AND graph distance >= 4
    (1-2, 1-3, 1-4 excluded);
  * types carry AutoDock4.1-like parameters (Rii, eps, vol, solpar) [ext];
    donor-H (HD) x acceptor pairs use a 12-10 H-bond potential, every other
    pair 12-6; the FE weights are folded into cA, cB;
  * charges ~ N(0, 0.25) e, re-centred to a neutral ligand;
  * reference coordinates are centred at the centroid (rotation centre).

Grid recipe: a pseudo-receptor of randomly placed atoms around a central
spherical pocket; maps are Gaussian-smoothed atom densities (repulsive core
minus attractive shell for type maps, smoothed charge potential for the
electrostatic map, smoothed density for desolvation), capped at +cap.
"""
from __future__ import annotations

import dataclasses
from dataclasses import dataclass, field

import numpy as np

# --------------------------------------------------------------------------
# Force-field constants (AutoDock4.2 values recalled [ext];
# both sides receive them as inputs, parity never depends on their values).
# --------------------------------------------------------------------------
FE_COEFF_VDW = 0.1662
FE_COEFF_HBOND = 0.1209
FE_COEFF_ESTAT = 0.1406
FE_COEFF_DESOLV = 0.1322


@dataclass
class FFParams:
    """Mirror of `ad_ff_params` in include/ad.h (same field order)."""
    smooth: float = 0.5            # A, width of the flat band around r0
    cut_vdw: float = 8.0           # A, vdW / H-bond cutoff (strict <)
    cut_el: float = 20.48          # A, electrostatics / desolvation cutoff
    el_rmin: float = 0.01          # A, floor on r in electrostatics
    diel_A: float = -8.5525        # Mehler-Solmajer dielectric
    diel_B: float = 78.4 + 8.5525
    diel_k: float = 7.7839
    diel_lambda: float = 0.003627
    coeff_el: float = 332.06363 * FE_COEFF_ESTAT
    coeff_ds: float = FE_COEFF_DESOLV
    qasp: float = 0.01097
    sigma_ds: float = 3.6
    w_out: float = 21.0            # kcal/mol per (grid unit)^2 outside the grid

    def as_array(self) -> np.ndarray:
        return np.array(dataclasses.astuple(self), dtype=np.float32)


# type name -> (Rii [A], eps [kcal/mol], vol [A^3], solpar, role, Rhb, eps_hb)
# role: 0 plain, 1 donor hydrogen, 2 acceptor
TYPE_PARAMS = {
    "C":  (4.00, 0.150, 33.5103, -0.00143, 0, 0.0, 0.0),
    "A":  (4.00, 0.150, 33.5103, -0.00052, 0, 0.0, 0.0),
    "N":  (3.50, 0.160, 22.4493, -0.00162, 0, 0.0, 0.0),
    "NA": (3.50, 0.160, 22.4493, -0.00162, 2, 1.9, 5.0),
    "OA": (3.20, 0.200, 17.1573, -0.00251, 2, 1.9, 5.0),
    "SA": (4.00, 0.200, 33.5103, -0.00214, 2, 2.5, 1.0),
    "HD": (2.00, 0.020, 0.0000, 0.00051, 1, 0.0, 0.0),
    "Cl": (4.09, 0.276, 35.8235, -0.00110, 0, 0.0, 0.0),
}

def pair_coefficients(names, params=None) -> np.ndarray:
    """Type-pair table [nt, nt, 5] = (cA, cB, r0, m, n) of the AD4 pair forms [ext]:
    donor-H x acceptor pairs 12-10 at (Rhb, eps_hb) of the acceptor, every other
    pair 12-6 at R = (R_i + R_j) / 2, eps = sqrt(eps_i eps_j); cA = fe eps r0^m n /
    (m - n), cB = fe eps r0^n m / (m - n) (minimum -fe eps at r0); FE weights folded
    in.  An input table (the ABI's tp_coef), not method arithmetic."""
    params = TYPE_PARAMS if params is None else params
    nt = len(names)
    tp = np.zeros((nt, nt, 5), dtype=np.float64)
    for a, na in enumerate(names):
        for b, nb in enumerate(names):
            Ra, ea, _, _, rola, Rhba, ehba = params[na]
            Rb, eb, _, _, rolb, Rhbb, ehbb = params[nb]
            if (rola, rolb) in ((1, 2), (2, 1)):
                r0, eps = (Rhbb, ehbb) if rola == 1 else (Rhba, ehba)
                m, n = 12.0, 10.0
                fe = FE_COEFF_HBOND
            else:
                r0, eps = 0.5 * (Ra + Rb), np.sqrt(ea * eb)
                m, n = 12.0, 6.0
                fe = FE_COEFF_VDW
            cA = fe * eps * r0 ** m * n / (m - n)
            cB = fe * eps * r0 ** n * m / (m - n)
            tp[a, b] = (cA, cB, r0, m, n)
    return tp


TYPESETS = {
    3: ["C", "OA", "HD"],
    6: ["C", "A", "N", "NA", "OA", "HD"],
    8: ["C", "A", "N", "NA", "OA", "SA", "HD", "Cl"],
}


@dataclass
class Ligand:
    """Mirror of `ad_ligand_desc` (include/ad.h); all arrays host numpy."""
    ref_xyz: np.ndarray        # [N,3] f32, centred at the rotation centre
    atom_map: np.ndarray       # [N] i32, type-map index into the grid maps
    atom_type: np.ndarray      # [N] i32, intra type index 0..n_types-1
    charge: np.ndarray         # [N] f32
    tors_axis: np.ndarray      # [T,2] i32, (a fixed side, c moving side), root->leaf
    tors_moving: np.ndarray    # [T,N] u8 0/1
    pairs: np.ndarray          # [P,2] i32, i<j
    tp_coef: np.ndarray        # [nt,nt,5] f32: cA, cB, r0, m, n
    type_S: np.ndarray         # [nt] f32 solpar
    type_V: np.ndarray         # [nt] f32 volume
    type_names: list = field(default_factory=list)
    bonds: np.ndarray = None   # [N-1,2] i32 (generator bookkeeping, tests only)
    frag: np.ndarray = None    # [N] i32 rigid fragment id

    @property
    def n_atoms(self) -> int:
        return int(self.ref_xyz.shape[0])

    @property
    def n_tors(self) -> int:
        return int(self.tors_axis.shape[0])

    @property
    def n_pairs(self) -> int:
        return int(self.pairs.shape[0])

    @property
    def n_types(self) -> int:
        return int(self.type_S.shape[0])

    @property
    def n_genes(self) -> int:
        return 6 + self.n_tors


@dataclass
class Grid:
    """Mirror of `ad_grid_desc` + maps[n_maps][nz][ny][nx] (x fastest)."""
    nx: int
    ny: int
    nz: int
    spacing: float
    origin: np.ndarray          # [3] f32
    maps: np.ndarray            # [n_maps, nz, ny, nx] f32

    @property
    def n_maps(self) -> int:
        return int(self.maps.shape[0])


# --------------------------------------------------------------------------
# ligand generator
# --------------------------------------------------------------------------
def _random_unit(rng):
    v = rng.normal(size=3)
    return v / np.linalg.norm(v)


def _place_child(rng, xyz, nbrs, p, bond):
    """Propose a position for a new atom bonded to p (bond angle 109.5+-5)."""
    if not nbrs[p]:
        return xyz[p] + bond * _random_unit(rng)
    b0 = xyz[nbrs[p][0]] - xyz[p]
    b0 /= np.linalg.norm(b0)
    ang = np.deg2rad(109.5 + rng.uniform(-5.0, 5.0))
    # orthonormal frame around b0
    t = _random_unit(rng)
    t -= b0 * np.dot(t, b0)
    t /= np.linalg.norm(t)
    d = np.cos(ang) * b0 + np.sin(ang) * t
    return xyz[p] + bond * d


def _graph_dist(n, adj):
    dist = np.full((n, n), 10**6, dtype=np.int64)
    for s in range(n):
        dist[s, s] = 0
        frontier = [s]
        while frontier:
            nxt = []
            for u in frontier:
                for v in adj[u]:
                    if dist[s, v] > dist[s, u] + 1:
                        dist[s, v] = dist[s, u] + 1
                        nxt.append(v)
            frontier = nxt
    return dist


def _build_tree(rng, n_atoms, chainlike):
    for _attempt in range(200):
        xyz = np.zeros((n_atoms, 3))
        nbrs = [[] for _ in range(n_atoms)]
        bonds = []
        ok = True
        for k in range(1, n_atoms):
            placed = False
            for _try in range(60):
                cand = [i for i in range(k) if len(nbrs[i]) < 3]
                if not cand:
                    break
                if chainlike and rng.uniform() < 0.6:
                    p = cand[max(0, len(cand) - 1 - int(rng.integers(0, 3)))]
                else:
                    p = cand[int(rng.integers(0, len(cand)))]
                bond = 1.5 + rng.uniform(-0.05, 0.05)
                for _a in range(12):
                    x = _place_child(rng, xyz, nbrs, p, bond)
                    # bond angles with all existing bonds of p >= 100 deg
                    good = True
                    for q in nbrs[p]:
                        u = xyz[q] - xyz[p]
                        v = x - xyz[p]
                        c = np.dot(u, v) / (np.linalg.norm(u) * np.linalg.norm(v))
                        if c > np.cos(np.deg2rad(100.0)):
                            good = False
                            break
                    if not good:
                        continue
                    d = np.linalg.norm(xyz[:k] - x, axis=1)
                    d[p] = 99.0
                    near = set(nbrs[p])  # 1-3 neighbours
                    lim = np.where([i in near for i in range(k)], 2.3, 2.9)
                    if np.all(d >= lim):
                        placed = True
                        break
                if placed:
                    xyz[k] = x
                    nbrs[p].append(k)
                    nbrs[k].append(p)
                    bonds.append((p, k))
                    break
            if not placed:
                ok = False
                break
        if ok:
            return xyz, nbrs, np.array(bonds, dtype=np.int32)
    raise RuntimeError("could not grow a ligand tree")


def make_ligand(seed: int, n_atoms: int, n_tors: int, n_types: int,
                chainlike: bool = False) -> Ligand:
    """Seeded random ligand (recipe in the module docstring)."""
    rng = np.random.default_rng(seed)
    names = TYPESETS[n_types]
    for _attempt in range(100):
        xyz, nbrs, bonds = _build_tree(rng, n_atoms, chainlike)
        deg = np.array([len(a) for a in nbrs])
        cand = [e for e, (u, v) in enumerate(bonds) if deg[u] >= 2 and deg[v] >= 2]
        if len(cand) >= n_tors:
            break
    else:
        raise RuntimeError("not enough non-terminal bonds for the torsion count")
    rot = sorted(rng.choice(len(cand), size=n_tors, replace=False).tolist()) if n_tors else []
    rot_edges = [tuple(int(x) for x in bonds[cand[r]]) for r in rot]
    rot_set = set(rot_edges) | set((v, u) for u, v in rot_edges)

    # rigid fragments: components after cutting the rotatable bonds
    frag = -np.ones(n_atoms, dtype=np.int32)
    nf = 0
    for s in range(n_atoms):
        if frag[s] >= 0:
            continue
        stack = [s]
        frag[s] = nf
        while stack:
            u = stack.pop()
            for v in nbrs[u]:
                if frag[v] < 0 and (u, v) not in rot_set:
                    frag[v] = nf
                    stack.append(v)
        nf += 1
    # torsion tree over fragments; root = the most central fragment
    fadj = [[] for _ in range(nf)]
    for u, v in rot_edges:
        fadj[frag[u]].append((frag[v], (u, v)))
        fadj[frag[v]].append((frag[u], (v, u)))

    def ecc(f0):
        seen = {f0: 0}
        fr = [f0]
        while fr:
            nx = []
            for f in fr:
                for g, _ in fadj[f]:
                    if g not in seen:
                        seen[g] = seen[f] + 1
                        nx.append(g)
            fr = nx
        return max(seen.values())
    root = min(range(nf), key=lambda f: (ecc(f), f))

    # orient torsions a (root side) -> c (moving side), BFS order root->leaf
    tors = []
    seen = {root}
    fr = [root]
    while fr:
        nx = []
        for f in fr:
            for g, (u, v) in sorted(fadj[f], key=lambda t: t[1]):
                if g not in seen:
                    seen.add(g)
                    tors.append((u, v))
                    nx.append(g)
        fr = nx
    adj = [list(a) for a in nbrs]
    moving = np.zeros((n_tors, n_atoms), dtype=np.uint8)
    for b, (a, c) in enumerate(tors):
        stack = [c]
        moving[b, c] = 1
        while stack:
            u = stack.pop()
            for v in adj[u]:
                if v != a and not moving[b, v]:
                    moving[b, v] = 1
                    stack.append(v)

    # types: leaves may be donor H bonded to N / OA; the rest heavy types
    heavy = [t for t in names if TYPE_PARAMS[t][4] != 1]
    has_hd = "HD" in names
    atype = np.array([heavy[int(rng.integers(0, len(heavy)))] for _ in range(n_atoms)], dtype=object)
    if has_hd:
        leaves = [i for i in range(n_atoms) if deg[i] == 1]
        rng.shuffle(leaves)
        n_hd = max(1, len(leaves) // 4)
        donors = [t for t in ("N", "OA") if t in names] or ["OA"]
        for i in leaves[:n_hd]:
            atype[i] = "HD"
            p = nbrs[i][0]
            if atype[p] not in donors:
                atype[p] = donors[int(rng.integers(0, len(donors)))]
        # make sure at least one acceptor exists
        acc = [t for t in names if TYPE_PARAMS[t][4] == 2]
        if acc and not any(TYPE_PARAMS[t][4] == 2 for t in atype):
            cands = [i for i in range(n_atoms) if atype[i] != "HD"]
            atype[cands[int(rng.integers(0, len(cands)))]] = acc[0]
    # HD atoms never sit on an axis atom (they are leaves), fine for torsions.
    atom_type = np.array([names.index(t) for t in atype], dtype=np.int32)

    q = rng.normal(0.0, 0.25, size=n_atoms)
    q -= q.mean()

    dist = _graph_dist(n_atoms, adj)
    ii, jj = np.triu_indices(n_atoms, k=1)
    keep = (frag[ii] != frag[jj]) & (dist[ii, jj] >= 4)
    pairs = np.stack([ii[keep], jj[keep]], axis=1).astype(np.int32)

    xyz = xyz - xyz.mean(axis=0)

    tp = pair_coefficients(names)
    return Ligand(
        ref_xyz=xyz.astype(np.float32),
        atom_map=atom_type.copy(),
        atom_type=atom_type,
        charge=q.astype(np.float32),
        tors_axis=np.array(tors, dtype=np.int32).reshape(n_tors, 2),
        tors_moving=moving,
        pairs=pairs,
        tp_coef=tp.astype(np.float32),
        type_S=np.array([TYPE_PARAMS[t][3] for t in names], dtype=np.float32),
        type_V=np.array([TYPE_PARAMS[t][2] for t in names], dtype=np.float32),
        type_names=list(names),
        bonds=bonds,
        frag=frag,
    )


# --------------------------------------------------------------------------
# grid generator
# --------------------------------------------------------------------------
def make_grid(seed: int, n_points: int, type_names, n_receptor: int,
              spacing: float = 0.375, pocket_radius: float | None = None,
              cap: float = 500.0) -> Grid:
    """Seeded pseudo-receptor maps, grid centred at the world origin."""
    from scipy.ndimage import gaussian_filter

    rng = np.random.default_rng(seed)
    n = n_points
    h = spacing
    half = 0.5 * h * (n - 1)
    origin = np.array([-half, -half, -half], dtype=np.float64)
    if pocket_radius is None:
        pocket_radius = 0.27 * 2 * half
    margin = 6.0
    lo, hi = -half - margin, half + margin
    pts = []
    while len(pts) < n_receptor:
        p = rng.uniform(lo, hi, size=(n_receptor, 3))
        p = p[np.linalg.norm(p, axis=1) > pocket_radius]
        pts.extend(p.tolist())
    rec = np.array(pts[:n_receptor])
    rq = rng.normal(0.0, 0.3, size=n_receptor)
    rkind = rng.integers(0, 3, size=n_receptor)  # 0 carbon-like, 1 donor, 2 acceptor

    pad = int(np.ceil(margin / h)) + 2
    m = n + 2 * pad
    gpos = (rec - origin) / h + pad
    idx = np.floor(gpos).astype(np.int64)
    f = gpos - idx

    def splat(weights):
        g = np.zeros((m, m, m))
        for dz in (0, 1):
            for dy in (0, 1):
                for dx in (0, 1):
                    w = ((f[:, 0] if dx else 1 - f[:, 0]) * (f[:, 1] if dy else 1 - f[:, 1])
                         * (f[:, 2] if dz else 1 - f[:, 2])) * weights
                    ix = np.clip(idx[:, 0] + dx, 0, m - 1)
                    iy = np.clip(idx[:, 1] + dy, 0, m - 1)
                    iz = np.clip(idx[:, 2] + dz, 0, m - 1)
                    np.add.at(g, (iz, iy, ix), w)
        return g

    def smooth(g, sigma_a):
        return gaussian_filter(g, sigma=sigma_a / h, mode="constant")[pad:pad + n, pad:pad + n, pad:pad + n]

    ones = np.ones(n_receptor)
    dens = splat(ones)
    rep = smooth(dens, 0.9)
    att = smooth(dens, 2.2)
    don = smooth(splat((rkind == 1).astype(float)), 1.6)
    acc = smooth(splat((rkind == 2).astype(float)), 1.6)
    # normalise so that one isolated receptor atom gives a unit peak
    def peak(sigma_a):
        return (2.0 * np.pi * (sigma_a / h) ** 2) ** -1.5
    rep /= peak(0.9)
    att /= peak(2.2)
    don /= peak(1.6)
    acc /= peak(1.6)

    maps = []
    for t in type_names:
        R, eps, vol, sol, role, Rhb, ehb = TYPE_PARAMS[t]
        v = 60.0 * eps * (R / 4.0) ** 6 * rep - 4.0 * eps * (R / 4.0) ** 3 * att
        if role == 1:
            v -= 1.5 * acc
        elif role == 2:
            v -= 1.2 * don
        maps.append(np.minimum(v, cap))
    el = smooth(splat(rq), 1.5)
    el = 8.0 * el / max(np.abs(el).max(), 1e-12)
    ds = smooth(dens, 3.6)
    ds = 0.8 * ds / max(ds.max(), 1e-12)
    maps.append(np.clip(el, -cap, cap))
    maps.append(np.minimum(ds, cap))
    arr = np.stack(maps).astype(np.float32)
    return Grid(nx=n, ny=n, nz=n, spacing=float(h), origin=origin.astype(np.float32), maps=arr)


# --------------------------------------------------------------------------
# genotypes
# --------------------------------------------------------------------------
def make_genotypes(seed: int, n_poses: int, n_tors: int, grid: Grid,
                   stride: int | None = None, frac: float = 0.5) -> np.ndarray:
    """Start genotypes [n_poses, stride] f32 (SURVEY §8(d) config 1 recipe).

    genes 0..2 translation in grid units, uniform over the central `frac` of the
    grid; 3..5 (phi, theta, alpha) degrees with theta = acos(1-2U) (uniform
    axis on the sphere); 6.. torsions U[-180,180).  Padding columns are 0.
    """
    rng = np.random.default_rng(seed)
    G = 6 + n_tors
    stride = stride or G
    out = np.zeros((n_poses, stride), dtype=np.float32)
    for k, nk in enumerate((grid.nx, grid.ny, grid.nz)):
        c = 0.5 * (nk - 1)
        out[:, k] = rng.uniform(c - 0.5 * frac * (nk - 1), c + 0.5 * frac * (nk - 1), size=n_poses)
    out[:, 3] = rng.uniform(0.0, 360.0, size=n_poses)
    out[:, 4] = np.degrees(np.arccos(1.0 - 2.0 * rng.uniform(size=n_poses)))
    out[:, 5] = rng.uniform(0.0, 360.0, size=n_poses)
    if n_tors:
        out[:, 6:G] = rng.uniform(-180.0, 180.0, size=(n_poses, n_tors))
    return out


# --------------------------------------------------------------------------
# configs
# --------------------------------------------------------------------------
@dataclass
class Workload:
    name: str
    grid: Grid
    ligands: list
    genes: np.ndarray           # [n_poses, stride]
    pose_ligand: np.ndarray     # [n_poses] i32 (index into ligands)
    runs: int
    pop: int
    iters: int
    ff: FFParams = field(default_factory=FFParams)

    @property
    def n_poses(self) -> int:
        return int(self.genes.shape[0])


CONFIGS = {
    1: dict(name="config1-tiny", n_atoms=12, n_tors=2, n_types=3, grid=32, receptor=400,
            runs=1, pop=256, iters=1),
    2: dict(name="config2-druglike", n_atoms=40, n_tors=8, n_types=6, grid=60, receptor=2000,
            runs=20, pop=150, iters=300),
    3: dict(name="config3-large", n_atoms=110, n_tors=32, n_types=8, grid=96, receptor=8000,
            runs=100, pop=150, iters=300),
}


def make_config(cfg: int, replica: int = 0, runs: int | None = None, pop: int | None = None,
                iters: int | None = None, stride: int | None = None) -> Workload:
    """Configs 1-3 as concrete seeded inputs (seed = 1000*config + replica)."""
    c = CONFIGS[cfg]
    seed = 1000 * cfg + replica
    lig = make_ligand(seed, c["n_atoms"], c["n_tors"], c["n_types"], chainlike=(cfg == 3))
    grid = make_grid(seed + 100, c["grid"], lig.type_names, c["receptor"])
    runs = runs or c["runs"]
    pop = pop or c["pop"]
    n = runs * pop
    genes = make_genotypes(seed + 200, n, lig.n_tors, grid, stride=stride)
    return Workload(name=c["name"], grid=grid, ligands=[lig], genes=genes,
                    pose_ligand=np.zeros(n, dtype=np.int32), runs=runs, pop=pop,
                    iters=iters or c["iters"])


class ScreenSpec:
    """Config 5 as a lazy recipe: the receptor grid and the per-ligand size draws
    up front; ligand k and its start genotypes generated on demand (a rank of a
    sharded screen builds only its own ligands).  Seeds as in make_screen."""

    def __init__(self, n_ligands: int = 8192, runs: int = 20, pop: int = 16, iters: int = 300,
                 replica: int = 0, stride: int = 40):
        self.seed = 5000 + replica
        self.n_ligands, self.runs, self.pop, self.iters, self.stride = n_ligands, runs, pop, iters, stride
        rng = np.random.default_rng(self.seed)
        self.sizes = []
        for _ in range(n_ligands):
            n = int(rng.integers(20, 111))
            t = int(rng.integers(0, min(32, n // 3) + 1))
            self.sizes.append((n, t))
        self.grid = make_grid(self.seed + 100, 60, TYPESETS[8], 2000)
        self.name = "config5-screen"

    def ligand(self, k: int) -> Ligand:
        n, t = self.sizes[k]
        return make_ligand(self.seed * 100003 + k, n, t, 8, chainlike=(n > 80))

    def genes(self, k: int) -> np.ndarray:
        """Start genotypes [runs * pop, stride] of ligand k (run-major)."""
        return make_genotypes(self.seed + 7 * k + 1, self.runs * self.pop, self.sizes[k][1], self.grid,
                              stride=self.stride)

    def n_pairs(self, k: int) -> float:
        """Intra-pair count ESTIMATE from the size draw (for sharding before the
        ligands exist; only relative costs matter): pairs between the T + 1 rigid
        fragments, ~ 0.4 n^2 (1 - 1 / (T + 1))."""
        n, t = self.sizes[k]
        return 0.4 * n * n * (1.0 - 1.0 / (t + 1))


def make_screen(n_ligands: int = 8192, runs: int = 20, pop: int = 16, iters: int = 300,
                replica: int = 0, stride: int = 40) -> Workload:
    """Config 5: heterogeneous screen over the config-2 receptor with 8 types
    (every ligand and genotype materialised; ScreenSpec is the lazy form)."""
    spec = ScreenSpec(n_ligands, runs, pop, iters, replica, stride)
    ligs = [spec.ligand(k) for k in range(n_ligands)]
    genes = np.concatenate([spec.genes(k) for k in range(n_ligands)]) if n_ligands else \
        np.zeros((0, stride), dtype=np.float32)
    pl = np.repeat(np.arange(n_ligands, dtype=np.int32), runs * pop)
    return Workload(name=spec.name, grid=spec.grid, ligands=ligs, genes=genes,
                    pose_ligand=pl, runs=runs, pop=pop, iters=iters)


def make_reduction_partials(seed: int, n_blocks: int, P: int, C: int, dist: str) -> np.ndarray:
    """Config 4: per-block partials [n_blocks, P, C] f32.

    dist: 'uniform' U(-1,1); 'logmag' log-uniform magnitudes 1e-4..1e4 with a
    random sign (cancellation-heavy)."""
    rng = np.random.default_rng(seed)
    if dist == "uniform":
        x = rng.uniform(-1.0, 1.0, size=(n_blocks, P, C))
    elif dist == "logmag":
        x = 10.0 ** rng.uniform(-4.0, 4.0, size=(n_blocks, P, C))
        x *= rng.choice([-1.0, 1.0], size=x.shape)
    else:
        raise ValueError(dist)
    return x.astype(np.float32)
