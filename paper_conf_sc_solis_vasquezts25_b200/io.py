"""Real docking inputs: AutoGrid maps and PDBQT ligands.

The paper's runs read receptor maps listed by an AutoGrid field file and a
ligand in PDBQT format (the artifact command P:L520-521:
``-ffile protein.maps.fld -lfile ligand.pdbqt``).  This module turns such files
into the plain arrays the C ABI takes (``synth.Grid`` / ``synth.Ligand``, the
mirrors of ``ad_grid_desc`` / ``ad_ligand_desc`` in include/ad.h), and writes
them back (for round-trip tests and for exporting synthetic workloads).  It is
host-side input handling: no pose building, energies or search happen here.

Formats (AutoDock4 conventions [ext], recalled, not in the paper):

* ``.map``: 6 header lines (GRID_PARAMETER_FILE, GRID_DATA_FILE, MACROMOLECULE,
  SPACING h, NELEMENTS nx ny nz (even), CENTER cx cy cz), then (nx+1)(ny+1)(nz+1)
  values, x fastest, then y, then z.  Point (i, j, k) sits at CENTER - h*NELEMENTS/2
  + h*(i, j, k).
* ``.maps.fld``: AVS field header; ``dim1..3`` = points per axis, ``label=``
  per component and ``variable n file=NAME filetype=ascii skip=6`` per map.  The
  type maps come first, then the electrostatic (``e``) and desolvation (``d``)
  maps -- the ABI's map order (include/ad.h: maps 0..n-3 type maps, n-2 elec,
  n-1 desolvation).
* ``.pdbqt``: ATOM/HETATM records (x, y, z in columns 31-54; then occupancy,
  B-factor, partial charge, AutoDock type), ROOT/ENDROOT, BRANCH a b /
  ENDBRANCH a b (a = serial of the parent-side atom, b = the first atom of the
  branch), TORSDOF.  Torsion b of the ABI = the BRANCH lines in file order
  (depth-first = root -> leaf, Z13), axis (a, b), moving set = the atoms inside
  the BRANCH block (nested branches included); rigid fragments = ROOT and each
  BRANCH's own atoms; bonds = the CONECT records when the file has them, else
  inferred from covalent radii; intramolecular pairs: different rigid fragment and graph distance >= 4
  (Z9, as the synthetic generator); rotation centre = the centroid (Z22).

The AD4.1 type parameters below are recalled AutoDock values [ext] (SURVEY
Appendix B lists the same ones for C, OA, N, HD); like every force-field
constant they are inputs to both the CUDA path and the oracle, so parity does
not depend on them.
"""
from __future__ import annotations

import os
import re

import numpy as np

from .synth import TYPE_PARAMS, Grid, Ligand, pair_coefficients

# AD4.1 bound parameters [ext]: type -> (Rii [A], eps [kcal/mol], vol [A^3], solpar,
# role (0 plain, 1 donor H, 2 acceptor), Rhb [A], eps_hb) -- the synth.TYPE_PARAMS layout
AD4_PARAMS = dict(TYPE_PARAMS)
AD4_PARAMS.update({
    "H":  (2.00, 0.020, 0.0000, 0.00051, 0, 0.0, 0.0),
    "HS": (2.00, 0.020, 0.0000, 0.00051, 1, 0.0, 0.0),
    "NS": (3.50, 0.160, 22.4493, -0.00162, 2, 1.9, 5.0),
    "OS": (3.20, 0.200, 17.1573, -0.00251, 2, 1.9, 5.0),
    "F":  (3.09, 0.080, 15.4480, -0.00110, 0, 0.0, 0.0),
    "Mg": (1.30, 0.875, 1.5600, -0.00110, 0, 0.0, 0.0),
    "P":  (4.20, 0.200, 38.7924, -0.00110, 0, 0.0, 0.0),
    "S":  (4.00, 0.200, 33.5103, -0.00214, 0, 0.0, 0.0),
    "Ca": (1.98, 0.550, 2.7700, -0.00110, 0, 0.0, 0.0),
    "Mn": (1.30, 0.875, 2.1400, -0.00110, 0, 0.0, 0.0),
    "Fe": (1.30, 0.010, 1.8400, -0.00110, 0, 0.0, 0.0),
    "Zn": (1.48, 0.550, 1.7000, -0.00110, 0, 0.0, 0.0),
    "Br": (4.33, 0.389, 42.5661, -0.00110, 0, 0.0, 0.0),
    "I":  (4.72, 0.550, 55.0585, -0.00110, 0, 0.0, 0.0),
})
for _upper, _t in (("CL", "Cl"), ("BR", "Br"), ("MG", "Mg"), ("CA", "Ca"), ("MN", "Mn"), ("FE", "Fe"), ("ZN", "Zn")):
    AD4_PARAMS[_upper] = AD4_PARAMS[_t]

# covalent radii [A] by element (bond inference; PDBQT carries no bonds) [ext]
_COV = {"H": 0.31, "C": 0.76, "N": 0.71, "O": 0.66, "S": 1.05, "P": 1.07, "F": 0.57, "Cl": 1.02, "Br": 1.20,
        "I": 1.39, "Mg": 1.41, "Ca": 1.76, "Mn": 1.39, "Fe": 1.32, "Zn": 1.22}
_ELEMENT = {"A": "C", "C": "C", "N": "N", "NA": "N", "NS": "N", "OA": "O", "OS": "O", "O": "O", "SA": "S",
            "S": "S", "H": "H", "HD": "H", "HS": "H", "P": "P", "F": "F", "Cl": "Cl", "CL": "Cl", "Br": "Br",
            "BR": "Br", "I": "I", "Mg": "Mg", "MG": "Mg", "Ca": "Ca", "CA": "Ca", "Mn": "Mn", "MN": "Mn",
            "Fe": "Fe", "FE": "Fe", "Zn": "Zn", "ZN": "Zn"}
BOND_TOL = 1.15  # bonded if d <= BOND_TOL * (r_i + r_j)


class FormatError(ValueError):
    """A malformed map / field / PDBQT file (message names the file and line)."""


# ----------------------------------------------------------------------------- maps
def read_map(path):
    """One AutoGrid map -> (header dict, values [nz, ny, nx] float32)."""
    with open(path) as f:
        lines = f.read().split("\n")
    hdr = {}
    k = 0
    while k < len(lines) and lines[k].split() and re.fullmatch(r"[A-Z][A-Z_]*", lines[k].split()[0]):
        key, *vals = lines[k].split()
        hdr[key] = vals
        k += 1
    try:
        h = float(hdr["SPACING"][0])
        ne = [int(v) for v in hdr["NELEMENTS"]]
        center = [float(v) for v in hdr["CENTER"]]
    except (KeyError, IndexError, ValueError) as e:
        raise FormatError(f"{path}: missing or bad SPACING / NELEMENTS / CENTER header ({e})")
    if len(ne) != 3 or any(n < 0 for n in ne) or len(center) != 3:
        raise FormatError(f"{path}: NELEMENTS needs 3 non-negative counts and CENTER 3 coordinates")
    nx, ny, nz = (n + 1 for n in ne)
    vals = np.array([float(v) for v in " ".join(lines[k:]).split()], dtype=np.float64)
    if vals.size != nx * ny * nz:
        raise FormatError(f"{path}: {vals.size} values, NELEMENTS {ne} needs {nx * ny * nz}")
    out = {"spacing": h, "nelements": ne, "center": center, "points": (nx, ny, nz),
           "origin": [center[d] - h * ne[d] / 2.0 for d in range(3)]}
    return out, vals.reshape(nz, ny, nx).astype(np.float32)


def read_fld(path):
    """An AutoGrid field file and the maps it lists -> (Grid, type-map names).

    The Grid's maps are ordered type maps (file order), electrostatic, desolvation
    (the ABI's order), whatever their order in the field file."""
    base = os.path.dirname(os.path.abspath(path))
    dims, variables = {}, []
    with open(path) as f:
        for ln, line in enumerate(f, 1):
            body = line.split("#", 1)[0].strip()
            if not body:
                continue
            if body.startswith("dim") and "=" in body:
                key, val = body.split("=", 1)
                dims[key.strip()] = int(val.split()[0])
            elif body.startswith("variable"):
                fields = dict(kv.split("=", 1) for kv in body.split()[2:] if "=" in kv)
                if "file" not in fields:
                    raise FormatError(f"{path}:{ln}: variable line without file=")
                variables.append(fields["file"])
    if not variables:
        raise FormatError(f"{path}: no variable lines")
    type_maps, elec, desolv = [], None, None
    for fn in variables:
        parts = os.path.basename(fn).split(".")
        tag = parts[-2] if len(parts) >= 3 else ""
        if tag == "e":
            elec = fn
        elif tag == "d":
            desolv = fn
        else:
            type_maps.append((tag, fn))
    if elec is None or desolv is None or not type_maps:
        raise FormatError(f"{path}: needs type maps plus the .e.map and .d.map")
    maps, names, ref = [], [], None
    for name, fn in type_maps + [("e", elec), ("d", desolv)]:
        hdr, v = read_map(os.path.join(base, fn))
        if ref is None:
            ref = hdr
        elif (hdr["points"] != ref["points"] or abs(hdr["spacing"] - ref["spacing"]) > 1e-6 or
              any(abs(a - b) > 1e-4 for a, b in zip(hdr["center"], ref["center"]))):
            raise FormatError(f"{fn}: grid differs from {type_maps[0][1]}")
        maps.append(v)
        if name not in ("e", "d"):
            names.append(name)
    if dims and tuple(dims.get(f"dim{d}", p) for d, p in zip((1, 2, 3), ref["points"])) != ref["points"]:
        raise FormatError(f"{path}: dim1..3 {dims} disagree with the maps' {ref['points']}")
    nx, ny, nz = ref["points"]
    grid = Grid(nx=nx, ny=ny, nz=nz, spacing=float(ref["spacing"]),
                origin=np.array(ref["origin"], dtype=np.float32), maps=np.stack(maps).astype(np.float32))
    return grid, names


def write_maps(grid, type_names, prefix, receptor="receptor"):
    """Write `grid` as AutoGrid maps PREFIX.<type>.map, PREFIX.e.map, PREFIX.d.map and
    the field file PREFIX.maps.fld (NELEMENTS must be even: odd point counts)."""
    if len(type_names) != grid.n_maps - 2:
        raise ValueError("one name per type map")
    pts = (grid.nx, grid.ny, grid.nz)
    if any(p % 2 == 0 for p in pts):
        raise ValueError("AutoGrid maps have an odd number of points per axis (NELEMENTS even)")
    ne = [p - 1 for p in pts]
    h = float(grid.spacing)
    center = [float(grid.origin[d]) + h * ne[d] / 2.0 for d in range(3)]
    stem = os.path.basename(prefix)
    files = []
    for name, m in zip(list(type_names) + ["e", "d"], grid.maps):
        fn = f"{prefix}.{name}.map"
        with open(fn, "w") as f:
            f.write(f"GRID_PARAMETER_FILE {stem}.gpf\nGRID_DATA_FILE {stem}.maps.fld\n"
                    f"MACROMOLECULE {receptor}.pdbqt\nSPACING {h:.4f}\n"
                    f"NELEMENTS {ne[0]} {ne[1]} {ne[2]}\nCENTER {center[0]:.4f} {center[1]:.4f} {center[2]:.4f}\n")
            np.savetxt(f, np.asarray(m, np.float64).reshape(-1), fmt="%.6g")
        files.append(os.path.basename(fn))
    with open(f"{prefix}.maps.fld", "w") as f:
        f.write("# AVS field file\n#\n# AutoDock Atomic Affinity and Electrostatic Grids\n#\n")
        f.write(f"#SPACING {h:.4f}\n#NELEMENTS {ne[0]} {ne[1]} {ne[2]}\n")
        f.write(f"#CENTER {center[0]:.4f} {center[1]:.4f} {center[2]:.4f}\n#\n")
        f.write(f"ndim=3\ndim1={pts[0]}\ndim2={pts[1]}\ndim3={pts[2]}\nnspace=3\nveclen={len(files)}\n"
                "data=float\nfield=uniform\n")
        for k, name in enumerate(list(type_names) + ["Electrostatics", "Desolvation"], 1):
            lab = f"{name}-affinity" if k <= len(type_names) else name
            f.write(f"label={lab}\n")
        for k, fn in enumerate(files, 1):
            f.write(f"variable {k} file={fn} filetype=ascii skip=6\n")


# --------------------------------------------------------------------------- pdbqt
def _graph_dist(n, bonds):
    adj = [[] for _ in range(n)]
    for a, b in bonds:
        adj[a].append(b)
        adj[b].append(a)
    dist = np.full((n, n), np.iinfo(np.int32).max, dtype=np.int64)
    for s in range(n):
        dist[s, s] = 0
        fr = [s]
        while fr:
            nx = []
            for u in fr:
                for v in adj[u]:
                    if dist[s, v] > dist[s, u] + 1:
                        dist[s, v] = dist[s, u] + 1
                        nx.append(v)
            fr = nx
    return dist


def read_pdbqt(path, map_names, params=None):
    """A PDBQT ligand -> (Ligand, centroid [3] float64).

    map_names: the grid's type-map names (read_fld); atom_map indexes them.  The
    reference coordinates are centred at the centroid (Z22), which is returned so
    that genes (translation = (centroid - origin) / h, orientation 0, torsions 0)
    reproduce the file's conformation."""
    params = AD4_PARAMS if params is None else params
    xyz, q, types, serial = [], [], [], []
    frag_of, branches = [], []  # per atom: innermost open block; branches: [a_serial, b_serial, first_atom, end]
    stack = []  # open blocks: fragment ids (0 = ROOT)
    conect = []  # explicit bonds (serial pairs), if the file has CONECT records
    n_frag = 0
    in_root = False
    with open(path) as f:
        lines = f.readlines()
    for ln, line in enumerate(lines, 1):
        rec = line[:6].strip()
        if rec not in ("ATOM", "HETATM", "CONECT"):
            rec = line.split()[0] if line.split() else ""
        if rec == "ROOT":
            in_root = True
            stack = [0]
            n_frag = max(n_frag, 1)
        elif rec == "ENDROOT":
            in_root = False
        elif rec == "BRANCH":
            try:
                a, b = (int(v) for v in line.split()[1:3])
            except ValueError:
                raise FormatError(f"{path}:{ln}: bad BRANCH line")
            if not stack:
                raise FormatError(f"{path}:{ln}: BRANCH outside the torsion tree")
            branches.append([a, b, len(xyz), None, n_frag])
            stack.append(n_frag)
            n_frag += 1
        elif rec == "ENDBRANCH":
            a, b = (int(v) for v in line.split()[1:3])
            open_b = [br for br in branches if br[3] is None]
            if not open_b or (open_b[-1][0], open_b[-1][1]) != (a, b):
                raise FormatError(f"{path}:{ln}: ENDBRANCH {a} {b} does not close the innermost BRANCH")
            open_b[-1][3] = len(xyz)
            stack.pop()
        elif rec == "CONECT":
            try:
                ids = [int(line[k:k + 5]) for k in range(6, len(line.rstrip()), 5)]
            except ValueError:
                raise FormatError(f"{path}:{ln}: bad CONECT record")
            conect.extend((ids[0], o) for o in ids[1:])
        elif rec in ("ATOM", "HETATM"):
            if not stack and not in_root:
                raise FormatError(f"{path}:{ln}: atom outside ROOT / BRANCH")
            try:
                serial.append(int(line[6:11]))
                xyz.append([float(line[30:38]), float(line[38:46]), float(line[46:54])])
                tail = line[54:].split()
                q.append(float(tail[-2]))
                types.append(tail[-1])
            except (ValueError, IndexError):
                raise FormatError(f"{path}:{ln}: bad ATOM record")
            frag_of.append(stack[-1])
    if not xyz:
        raise FormatError(f"{path}: no atoms")
    if any(br[3] is None for br in branches):
        raise FormatError(f"{path}: unclosed BRANCH")
    n = len(xyz)
    xyz = np.array(xyz, dtype=np.float64)
    idx = {s: i for i, s in enumerate(serial)}
    if len(idx) != n:
        raise FormatError(f"{path}: duplicate atom serial numbers")
    for t in types:
        if t not in params:
            raise FormatError(f"{path}: unknown AutoDock type {t!r}")
        if t not in map_names and t.capitalize() not in map_names:
            raise FormatError(f"{path}: no grid map for type {t!r} (maps: {map_names})")
    # bonds: the CONECT records if present, else from covalent radii; plus every BRANCH axis
    if conect:
        try:
            bonds = set((min(idx[a], idx[b]), max(idx[a], idx[b])) for a, b in conect if a != b)
        except KeyError as e:
            raise FormatError(f"{path}: CONECT names a missing atom {e}")
    else:
        el = [_ELEMENT.get(t, "C") for t in types]
        rc = np.array([_COV.get(e, 0.76) for e in el])
        d = np.linalg.norm(xyz[:, None, :] - xyz[None, :, :], axis=-1)
        ii, jj = np.nonzero(np.triu(d <= BOND_TOL * (rc[:, None] + rc[None, :]), 1))
        bonds = set(zip(ii.tolist(), jj.tolist()))
    tors_axis, moving = [], np.zeros((len(branches), n), dtype=np.uint8)
    for k, (a, b, lo, hi, _) in enumerate(branches):
        if a not in idx or b not in idx:
            raise FormatError(f"{path}: BRANCH {a} {b} names a missing atom")
        ia, ib = idx[a], idx[b]
        if not (lo <= ib < hi) or (lo <= ia < hi):
            raise FormatError(f"{path}: BRANCH {a} {b}: {b} must be inside the branch and {a} outside")
        bonds.add((min(ia, ib), max(ia, ib)))
        tors_axis.append((ia, ib))
        moving[k, lo:hi] = 1
    # the rotatable bonds themselves are the only bonds between fragments
    frag = np.array(frag_of, dtype=np.int32)
    bonds = sorted(bonds)
    dist = _graph_dist(n, bonds)
    iu, ju = np.triu_indices(n, k=1)
    keep = (frag[iu] != frag[ju]) & (dist[iu, ju] >= 4)
    pairs = np.stack([iu[keep], ju[keep]], axis=1).astype(np.int32)
    names = []
    for t in types:
        if t not in names:
            names.append(t)
    atom_type = np.array([names.index(t) for t in types], dtype=np.int32)
    mapname = {m: k for k, m in enumerate(map_names)}
    atom_map = np.array([mapname[t] if t in mapname else mapname[t.capitalize()] for t in types], dtype=np.int32)
    centroid = xyz.mean(axis=0)
    lig = Ligand(
        ref_xyz=(xyz - centroid).astype(np.float32),
        atom_map=atom_map,
        atom_type=atom_type,
        charge=np.array(q, dtype=np.float32),
        tors_axis=np.array(tors_axis, dtype=np.int32).reshape(len(branches), 2),
        tors_moving=moving,
        pairs=pairs,
        tp_coef=pair_coefficients(names, params).astype(np.float32),
        type_S=np.array([params[t][3] for t in names], dtype=np.float32),
        type_V=np.array([params[t][2] for t in names], dtype=np.float32),
        type_names=names,
        bonds=np.array(bonds, dtype=np.int32).reshape(-1, 2),
        frag=frag,
    )
    return lig, centroid


def input_genes(lig_centroid, grid, n_tors, stride=None):
    """The genotype reproducing a PDBQT conformation: translation = the centroid in
    grid units, orientation (phi, theta, alpha) = 0, torsions = 0 (Z11)."""
    g = np.zeros(stride or (6 + n_tors), dtype=np.float32)
    g[:3] = (np.asarray(lig_centroid, np.float64) - np.asarray(grid.origin, np.float64)) / float(grid.spacing)
    return g


def write_pdbqt(lig, path, centroid=(0.0, 0.0, 0.0), resname="LIG", bonds=True):
    """Write a Ligand (torsion tree = tors_axis / tors_moving, listed root -> leaf)
    as PDBQT: ROOT = atoms no torsion moves, then nested BRANCH blocks; atoms are
    written in block order, so serial numbers follow that order; bonds=True adds
    CONECT records of lig.bonds (when known).  Returns the order (new position ->
    ligand atom index)."""
    n, T = lig.n_atoms, lig.n_tors
    mv = np.asarray(lig.tors_moving, bool)
    # parent torsion of each torsion: the smallest moving set strictly containing it
    parent = [-1] * T
    for b in range(T):
        best = -1
        for c in range(T):
            if c != b and mv[c][mv[b]].all() and mv[c].sum() > mv[b].sum():
                if best < 0 or mv[c].sum() < mv[best].sum():
                    best = c
        parent[b] = best
    owner = np.full(n, -1)  # innermost torsion moving each atom
    for a in range(n):
        cands = [b for b in range(T) if mv[b, a]]
        if cands:
            owner[a] = min(cands, key=lambda b: mv[b].sum())
    order = []
    out = []
    serial = {}

    def atom_line(a):
        serial[a] = len(order) + 1
        order.append(a)
        x, y, z = (np.asarray(lig.ref_xyz[a], np.float64) + np.asarray(centroid, np.float64)).tolist()
        t = lig.type_names[int(lig.atom_type[a])]
        el = _ELEMENT.get(t, "C")
        name = f"{el}{serial[a]}"[:4]
        return (f"ATOM  {serial[a]:5d} {name:<4s} {resname:3s} A   1    {x:8.3f}{y:8.3f}{z:8.3f}"
                f"  1.00  0.00    {float(lig.charge[a]):+6.3f} {t:<2s}")

    def emit(b):
        # atoms owned by b first (so the moving-side axis atom is inside), then children
        a_ax, c_ax = (int(v) for v in lig.tors_axis[b])
        own = [a for a in range(n) if owner[a] == b]
        own.sort(key=lambda a: (a != c_ax, a))
        body = [atom_line(a) for a in own]
        kids = [c for c in range(T) if parent[c] == b]
        head = len(out)
        out.append(None)  # BRANCH placeholder (needs the axis serials)
        out.extend(body)
        for c in kids:
            emit(c)
        out[head] = f"BRANCH {serial[a_ax]:3d} {serial[c_ax]:3d}"
        out.append(f"ENDBRANCH {serial[a_ax]:3d} {serial[c_ax]:3d}")

    out.append("ROOT")
    for a in range(n):
        if owner[a] < 0:
            out.append(atom_line(a))
    out.append("ENDROOT")
    for b in range(T):
        if parent[b] < 0:
            emit(b)
    out.append(f"TORSDOF {T}")
    if bonds and lig.bonds is not None:  # explicit bonds (the generator's tree), PDB CONECT records
        for a, b in np.asarray(lig.bonds).reshape(-1, 2).tolist():
            out.append(f"CONECT{serial[a]:5d}{serial[b]:5d}")
    with open(path, "w") as f:
        f.write(f"REMARK  {T} active torsions\n")
        f.write("\n".join(out) + "\n")
    return np.array(order, dtype=np.int32)
