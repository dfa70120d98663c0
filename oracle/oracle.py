"""ctypes front-end of the FP64 CPU oracle (oracle/ad_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py.  The product package never
imports this module.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "ad_oracle.c")
LIB = os.path.join(HERE, "libad_oracle.so")

AUX_EINTER, AUX_EINTRA, AUX_ABS_E, AUX_MARGIN_E, AUX_MARGIN_G, AUX_SENS_E, AUX_N = range(7)

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2, no fast-math, OpenMP)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-Wall", "-o", LIB, SRC, "-lm"]
        subprocess.check_call(cmd)
    return LIB


class Grid_(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("n_maps", C.c_int32),
                ("spacing", C.c_double), ("origin", C.c_double * 3), ("maps", C.c_void_p)]


class FF_(C.Structure):
    _fields_ = [(n, C.c_double) for n in ("smooth", "cut_vdw", "cut_el", "el_rmin", "diel_A", "diel_B", "diel_k",
                                          "diel_lambda", "coeff_el", "coeff_ds", "qasp", "sigma_ds", "w_out")]


class Lig_(C.Structure):
    _fields_ = [("n_atoms", C.c_int32), ("n_tors", C.c_int32), ("n_pairs", C.c_int32), ("n_types", C.c_int32),
                ("ref_xyz", C.c_void_p), ("atom_map", C.c_void_p), ("atom_type", C.c_void_p),
                ("charge", C.c_void_p), ("tors_axis", C.c_void_p), ("tors_moving", C.c_void_p),
                ("pairs", C.c_void_p), ("tp_coef", C.c_void_p), ("type_S", C.c_void_p), ("type_V", C.c_void_p)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(LIB)
            P = C.c_void_p
            L.ado_pose.argtypes = [P, P, P, P, P]
            L.ado_eval.argtypes = [P, P, P, P, P, P, P, P, P]
            L.ado_score.argtypes = [P, P, P, C.c_int32, P, C.c_int32, P, P, P, P, C.c_int32]
            L.ado_adadelta_step.argtypes = [C.c_int32, P, P, P, P, C.c_double, C.c_double]
            L.ado_local_search.argtypes = [P, P, P, C.c_int32, P, C.c_int32, C.c_int32, C.c_double, C.c_double,
                                           P, P, P, C.c_int32]
            L.ado_best_of_run.argtypes = [C.c_int32, C.c_int32, P, P]
            L.ado_exact_sum.argtypes = [P, C.c_int64, C.c_int64]
            L.ado_exact_sum.restype = C.c_double
            L.ado_rng.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32]
            L.ado_rng.restype = C.c_uint64
            L.ado_rng_mix.argtypes = [C.c_uint64]
            L.ado_rng_mix.restype = C.c_uint64
            L.ado_ga_generation.argtypes = [P, P, P, P, C.c_uint64, C.c_uint32, C.c_uint32]
            L.ado_ls_select.argtypes = [P, C.c_uint64, C.c_uint32, C.c_uint32, P]
            _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


class _Keep:
    """Holds the numpy arrays a ctypes struct points into."""

    def __init__(self):
        self.arrs = []

    def __call__(self, a, dtype):
        a = np.ascontiguousarray(a, dtype=dtype)
        self.arrs.append(a)
        return _ptr(a)


def _structs(lig, grid, ff):
    k = _Keep()
    g = Grid_(grid.nx, grid.ny, grid.nz, grid.n_maps, float(grid.spacing),
              (C.c_double * 3)(*[float(v) for v in grid.origin]), k(grid.maps, np.float32))
    f = FF_(*[float(v) for v in ff.as_array()])
    lg = Lig_(lig.n_atoms, lig.n_tors, lig.n_pairs, lig.n_types,
              k(lig.ref_xyz, np.float32), k(lig.atom_map, np.int32), k(lig.atom_type, np.int32),
              k(lig.charge, np.float32), k(lig.tors_axis.reshape(-1, 2), np.int32),
              k(lig.tors_moving.reshape(-1), np.uint8), k(lig.pairs.reshape(-1, 2), np.int32),
              k(lig.tp_coef, np.float32), k(lig.type_S, np.float32), k(lig.type_V, np.float32))
    return lg, g, f, k


def pose(lig, grid, genes_row) -> np.ndarray:
    """O-1 for one genotype (float64 input) -> X [N,3] float64."""
    lg, g, _f, keep = _structs(lig, grid, _dummy_ff())
    x = np.ascontiguousarray(genes_row, dtype=np.float64)
    X = np.zeros((lig.n_atoms, 3))
    T = np.zeros(3)
    lib().ado_pose(C.byref(lg), C.byref(g), _ptr(x), _ptr(X), _ptr(T))
    return X


def eval_one(lig, grid, ff, genes_row):
    """One pose in float64: (E, grad[G], aux[AUX_N], agrad[G], X[N,3])."""
    lg, g, f, keep = _structs(lig, grid, ff)
    x = np.ascontiguousarray(genes_row[:lig.n_genes], dtype=np.float64)
    E = np.zeros(1)
    gr = np.zeros(lig.n_genes)
    aux = np.zeros(AUX_N)
    ag = np.zeros(lig.n_genes)
    X = np.zeros((lig.n_atoms, 3))
    rc = lib().ado_eval(C.byref(lg), C.byref(g), C.byref(f), _ptr(x), _ptr(E), _ptr(gr), _ptr(aux), _ptr(ag), _ptr(X))
    assert rc == 0
    return float(E[0]), gr, aux, ag, X


def score(lig, grid, ff, genes: np.ndarray, threads: int = 0):
    """Batch of FP32 genotypes [n, stride]: E[n], grad[n, stride], aux[n, AUX_N], agrad[n, stride]."""
    lg, g, f, keep = _structs(lig, grid, ff)
    genes = np.ascontiguousarray(genes, dtype=np.float32)
    n, stride = genes.shape
    E = np.zeros(n)
    gr = np.zeros((n, stride))
    aux = np.zeros((n, AUX_N))
    ag = np.zeros((n, stride))
    rc = lib().ado_score(C.byref(lg), C.byref(g), C.byref(f), n, _ptr(genes), stride, _ptr(E), _ptr(gr), _ptr(aux),
                         _ptr(ag), threads or os.cpu_count())
    assert rc == 0, rc
    return E, gr, aux, ag


def local_search(lig, grid, ff, genes: np.ndarray, max_iters=300, rho=0.8, eps=0.01, threads: int = 0,
                 trace: bool = False):
    """O-6 from FP32 start genotypes [n, stride]: (best_genes, best_E) and, with
    trace=True, (E, A_E, S_E, margin_e, margin_g) of every step [n, max_iters, 5] as a third output."""
    lg, g, f, keep = _structs(lig, grid, ff)
    genes = np.ascontiguousarray(genes, dtype=np.float32)
    n, stride = genes.shape
    best = np.zeros((n, stride))
    bE = np.zeros(n)
    tE = np.zeros((n, max_iters, 5)) if trace else None
    rc = lib().ado_local_search(C.byref(lg), C.byref(g), C.byref(f), n, _ptr(genes), stride, max_iters, rho, eps,
                                _ptr(best), _ptr(bE), _ptr(tE) if trace else None, threads or os.cpu_count())
    assert rc == 0, rc
    return (best, bE, tE) if trace else (best, bE)


def adadelta_step(grad, eg2, ed2, genes, rho=0.8, eps=0.01):
    """One O-6 update in float64; returns (eg2, ed2, genes) new copies."""
    grad = np.ascontiguousarray(grad, dtype=np.float64)
    eg2 = np.array(eg2, dtype=np.float64)
    ed2 = np.array(ed2, dtype=np.float64)
    genes = np.array(genes, dtype=np.float64)
    lib().ado_adadelta_step(len(grad), _ptr(grad), _ptr(eg2), _ptr(ed2), _ptr(genes), rho, eps)
    return eg2, ed2, genes


def best_of_run(best_E, pop):
    best_E = np.ascontiguousarray(best_E, dtype=np.float64)
    out = np.zeros(len(best_E) // pop, dtype=np.int32)
    assert lib().ado_best_of_run(len(best_E), pop, _ptr(best_E), _ptr(out)) == 0
    return out


def exact_sum(x: np.ndarray) -> float:
    x = np.ascontiguousarray(x, dtype=np.float32).reshape(-1)
    return float(lib().ado_exact_sum(_ptr(x), x.size, 1))


class GA_(C.Structure):
    _fields_ = [("pop", C.c_int32), ("n_genes", C.c_int32), ("stride", C.c_int32), ("elitism", C.c_int32),
                ("cross_rate", C.c_float), ("mut_rate", C.c_float), ("tour_rate", C.c_float), ("ls_rate", C.c_float),
                ("dmov", C.c_float), ("dang", C.c_float)]


def ga_params(pop, n_genes, stride, elitism=1, cross_rate=0.8, mut_rate=0.02, tour_rate=0.6, ls_rate=0.8,
              dmov=16.0, dang=90.0):
    """NEXT-3 GA parameters (DESIGN.md 7b readings; dmov in grid units)."""
    return GA_(pop, n_genes, stride, elitism, cross_rate, mut_rate, tour_rate, ls_rate, dmov, dang)


def rng(seed, gen, run, ind, d) -> int:
    """The counter-based generator of the GA (oracle side)."""
    return int(lib().ado_rng(seed, gen, run, ind, d))


def ga_generation(prm, genes, energies, seed, gen, run):
    """One GA generation of one run: genes [pop, stride] f32, energies [pop] f32 -> new genes."""
    genes = np.ascontiguousarray(genes, dtype=np.float32)
    energies = np.ascontiguousarray(energies, dtype=np.float32)
    out = np.zeros_like(genes)
    assert lib().ado_ga_generation(C.byref(prm), _ptr(genes), _ptr(energies), _ptr(out), seed, gen, run) == 0
    return out


def ls_select(prm, seed, gen, run):
    sel = np.zeros(prm.pop, dtype=np.uint8)
    lib().ado_ls_select(C.byref(prm), seed, gen, run, _ptr(sel))
    return sel.astype(bool)


def _dummy_ff():
    from paper_conf_sc_solis_vasquezts25_b200.synth import FFParams
    return FFParams()
