"""Hand-built tiny inputs for oracle pins and GPU edge cases (no method arithmetic)."""
import numpy as np

from paper_conf_sc_solis_vasquezts25_b200.synth import FFParams, Grid, Ligand


def hand_ligand(xyz, tors_axis=(), moving=(), pairs=(), types=None, charges=None, tp=None, S=None, V=None):
    xyz = np.asarray(xyz, dtype=np.float32)
    N = len(xyz)
    T = len(tors_axis)
    types = np.zeros(N, np.int32) if types is None else np.asarray(types, np.int32)
    nt = int(types.max()) + 1
    if tp is None:
        tp = np.zeros((nt, nt, 5), np.float32)
        tp[..., 3] = 12.0
        tp[..., 4] = 6.0
        tp[..., 2] = 4.0
    mv = np.zeros((T, N), np.uint8)
    for b, m in enumerate(moving):
        mv[b, list(m)] = 1
    return Ligand(
        ref_xyz=xyz,
        atom_map=types.copy(),
        atom_type=types,
        charge=np.zeros(N, np.float32) if charges is None else np.asarray(charges, np.float32),
        tors_axis=np.asarray(tors_axis, np.int32).reshape(T, 2),
        tors_moving=mv,
        pairs=np.asarray(pairs, np.int32).reshape(-1, 2),
        tp_coef=np.asarray(tp, np.float32),
        type_S=np.zeros(nt, np.float32) if S is None else np.asarray(S, np.float32),
        type_V=np.zeros(nt, np.float32) if V is None else np.asarray(V, np.float32),
        type_names=[f"t{k}" for k in range(nt)],
    )


def const_grid(n=24, h=0.375, n_type_maps=1, value=0.0, center=True):
    half = 0.5 * h * (n - 1) if center else 0.0
    origin = np.array([-half, -half, -half], np.float32)
    maps = np.full((n_type_maps + 2, n, n, n), value, np.float32)
    return Grid(nx=n, ny=n, nz=n, spacing=h, origin=origin, maps=maps)


def affine_grid(coefs, n=16, h=0.5, origin=(-3.0, -2.5, -4.0)):
    """maps[m](u) = a_m + b_m . u  (u in grid units) for each (a_m, b_m) in coefs."""
    z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    maps = np.stack([a + b[0] * x + b[1] * y + b[2] * z for a, b in coefs]).astype(np.float32)
    return Grid(nx=n, ny=n, nz=n, spacing=h, origin=np.asarray(origin, np.float32), maps=maps)


def identity_genes(grid, point, n_tors):
    """Genes that place the rotation centre at `point` with identity orientation."""
    g = np.zeros(6 + n_tors)
    g[:3] = (np.asarray(point, float) - np.asarray(grid.origin, float)) / grid.spacing
    return g


def ff_default():
    return FFParams()


def f32(x):
    """Inputs (constants included) cross both boundaries as FP32."""
    return float(np.float32(x))
