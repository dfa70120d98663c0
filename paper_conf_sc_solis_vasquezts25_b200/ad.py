"""Python binding of libad (include/ad.h): argument marshalling only.

Every function named ``ad_*`` here forwards to the C entry point of the same
name; every step of the hot path runs in libad's CUDA kernels.  torch is used
for device memory and streams only.  There is no CPU fallback: if libad.so is
missing or no CUDA device is present, the calls raise.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AD_LIB", os.path.join(PKG, "libad.so"))  # AD_LIB: A/B builds

AD_OK, AD_ERR_INVALID_ARG, AD_ERR_LIMIT, AD_ERR_CUDA, AD_ERR_OOM, AD_ERR_STATE = 0, -1, -2, -3, -4, -5
AD_ENGINE_SIMT, AD_ENGINE_TC, AD_ENGINE_PAPER_BASELINE, AD_ENGINE_PAPER_TCEC, AD_ENGINE_TC_FP16 = 0, 1, 2, 3, 4
ENGINES = {"simt": AD_ENGINE_SIMT, "tc": AD_ENGINE_TC, "paper": AD_ENGINE_PAPER_BASELINE,
           "paper_tcec": AD_ENGINE_PAPER_TCEC, "tc_fp16": AD_ENGINE_TC_FP16}

# names exported by include/ad.h (tests check the .so exports all of them)
EXPORTS = ("ad_last_error", "ad_version", "ad_context_create", "ad_context_destroy", "ad_upload_grids",
           "ad_upload_ligand", "ad_free_ligand", "ad_set_launch_ligands", "ad_set_schedule_effort",
           "ad_score_poses", "ad_local_search", "ad_lga_run", "ad_reduce_blocks", "ad_sync", "ad_query",
           "ad_last_launch")


class AdError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"libad error {code}: {msg}")
        self.code = code


class GridDesc(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("n_maps", C.c_int32),
                ("spacing", C.c_float), ("origin", C.c_float * 3)]


class FFParams(C.Structure):
    _fields_ = [(n, C.c_float) for n in ("smooth", "cut_vdw", "cut_el", "el_rmin", "diel_A", "diel_B", "diel_k",
                                         "diel_lambda", "coeff_el", "coeff_ds", "qasp", "sigma_ds", "w_out")]


class LigandDesc(C.Structure):
    _fields_ = [("n_atoms", C.c_int32), ("n_tors", C.c_int32), ("n_pairs", C.c_int32), ("n_types", C.c_int32),
                ("ref_xyz", C.c_void_p), ("atom_map", C.c_void_p), ("atom_type", C.c_void_p), ("charge", C.c_void_p),
                ("tors_axis", C.c_void_p), ("tors_moving", C.c_void_p), ("pairs", C.c_void_p),
                ("tp_coef", C.c_void_p), ("type_S", C.c_void_p), ("type_V", C.c_void_p), ("ff", C.c_void_p)]


class LSParams(C.Structure):
    _fields_ = [("max_iters", C.c_int32), ("rho", C.c_float), ("eps", C.c_float), ("pop_per_run", C.c_int32),
                ("engine", C.c_int32), ("warps_per_cta", C.c_int32), ("trace", C.c_void_p),
                ("phase_cycles", C.c_void_p)]


class LGAParams(C.Structure):
    _fields_ = [("pop_size", C.c_int32), ("max_gens", C.c_int32), ("max_evals", C.c_int64), ("elitism", C.c_int32),
                ("cross_rate", C.c_float), ("mut_rate", C.c_float), ("tour_rate", C.c_float), ("ls_rate", C.c_float),
                ("dmov", C.c_float), ("dang", C.c_float), ("seed", C.c_uint64), ("ls", LSParams)]


_lock = threading.Lock()
_lib = None


def lib():
    """Load libad.so (fails loudly if it was not built)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; "
                                  f"g.build()'` (nvcc, sm_100a). There is no CPU fallback.")
            L = C.CDLL(LIB_PATH)
            P, I32 = C.c_void_p, C.c_int32
            L.ad_last_error.restype = C.c_char_p
            L.ad_version.restype = I32
            L.ad_context_create.argtypes = [I32, C.POINTER(C.c_void_p)]
            L.ad_context_destroy.argtypes = [P]
            L.ad_upload_grids.argtypes = [P, C.POINTER(GridDesc), P, I32, P]
            L.ad_upload_ligand.argtypes = [P, C.POINTER(LigandDesc), C.POINTER(I32)]
            L.ad_free_ligand.argtypes = [P, I32]
            L.ad_set_schedule_effort.argtypes = [P, I32]
            L.ad_set_launch_ligands.argtypes = [P, P, I32]
            L.ad_score_poses.argtypes = [P, I32, P, I32, P, I32, P, P, P, P]
            L.ad_local_search.argtypes = [P, I32, P, I32, P, I32, P, P, P, C.POINTER(LSParams), P]
            L.ad_reduce_blocks.argtypes = [P, I32, I32, I32, I32, P, P, P]
            L.ad_lga_run.argtypes = [P, I32, I32, P, I32, P, P, P, P, C.POINTER(LGAParams), P]
            L.ad_sync.argtypes = [P, P]
            L.ad_query.argtypes = [P, I32, C.POINTER(I32), C.POINTER(I32), C.POINTER(I32)]
            L.ad_last_launch.argtypes = [P, C.POINTER(I32), C.POINTER(I32), C.POINTER(I32)]
            for name in EXPORTS:
                if name not in ("ad_last_error", "ad_version"):
                    getattr(L, name).restype = I32
            _lib = L
    return _lib


def _check(rc):
    if rc != AD_OK:
        raise AdError(rc, lib().ad_last_error().decode())


def _dptr(t, dtype=None):
    """Device pointer of a CUDA tensor (or None -> NULL)."""
    if t is None:
        return None
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError("expected a CUDA torch.Tensor")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"expected {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return C.c_void_p(t.data_ptr())


def _stream(stream):
    import torch
    if stream is None:
        # the raw cudaStream_t of the current stream without building a Stream object
        # (torch.cuda.current_stream() costs ~3 us per call, a config-1 score call ~9 us)
        raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)
        if raw is not None:
            return C.c_void_p(raw(torch.cuda.current_device()))
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


# ---------------------------------------------------------------- raw C calls
def ad_version() -> int:
    return int(lib().ad_version())


def ad_context_create(device: int = 0):
    h = C.c_void_p()
    _check(lib().ad_context_create(device, C.byref(h)))
    return h


def ad_context_destroy(ctx) -> None:
    _check(lib().ad_context_destroy(ctx))


def ad_upload_grids(ctx, grid, stream=None) -> None:
    maps = np.ascontiguousarray(grid.maps, dtype=np.float32)
    d = GridDesc(grid.nx, grid.ny, grid.nz, maps.shape[0], float(grid.spacing),
                 (C.c_float * 3)(*[float(v) for v in grid.origin]))
    _check(lib().ad_upload_grids(ctx, C.byref(d), maps.ctypes.data_as(C.c_void_p), 0, _stream(stream)))


def ad_upload_ligand(ctx, lig, ff) -> int:
    keep = []

    def arr(a, dt):
        a = np.ascontiguousarray(a, dtype=dt)
        keep.append(a)
        return a.ctypes.data_as(C.c_void_p)

    f = FFParams(*[float(v) for v in ff.as_array()])
    d = LigandDesc(lig.n_atoms, lig.n_tors, lig.n_pairs, lig.n_types,
                   arr(lig.ref_xyz, np.float32), arr(lig.atom_map, np.int32), arr(lig.atom_type, np.int32),
                   arr(lig.charge, np.float32), arr(lig.tors_axis.reshape(-1, 2), np.int32),
                   arr(lig.tors_moving.reshape(-1), np.uint8), arr(lig.pairs.reshape(-1, 2), np.int32),
                   arr(lig.tp_coef, np.float32), arr(lig.type_S, np.float32), arr(lig.type_V, np.float32),
                   C.cast(C.pointer(f), C.c_void_p))
    out = C.c_int32()
    _check(lib().ad_upload_ligand(ctx, C.byref(d), C.byref(out)))
    return int(out.value)


def ad_free_ligand(ctx, lig: int) -> None:
    _check(lib().ad_free_ligand(ctx, lig))


def ad_set_launch_ligands(ctx, ids) -> None:
    a = np.ascontiguousarray(list(ids) if ids is not None else [], dtype=np.int32)
    _check(lib().ad_set_launch_ligands(ctx, a.ctypes.data_as(C.c_void_p) if a.size else None, int(a.size)))


def ad_set_schedule_effort(ctx, effort: int) -> None:
    _check(lib().ad_set_schedule_effort(ctx, int(effort)))


def ad_score_poses(ctx, lig, pose_ligand, genes, energy, grad=None, aux=None, stream=None) -> None:
    import torch
    n, stride = genes.shape
    _check(lib().ad_score_poses(ctx, lig, _dptr(pose_ligand, torch.int32), n, _dptr(genes, torch.float32), stride,
                                _dptr(energy, torch.float32), _dptr(grad, torch.float32), _dptr(aux, torch.float32),
                                _stream(stream)))


def ad_local_search(ctx, lig, pose_ligand, genes, best_energy, run_best=None, n_evals=None, *, max_iters=300,
                    rho=0.8, eps=0.01, pop_per_run=0, engine=AD_ENGINE_SIMT, warps_per_cta=0, trace=None,
                    phase_cycles=None, stream=None) -> None:
    import torch
    n, stride = genes.shape
    prm = LSParams(max_iters, rho, eps, pop_per_run, engine, warps_per_cta, _dptr(trace, torch.float32),
                   _dptr(phase_cycles, torch.int64))
    _check(lib().ad_local_search(ctx, lig, _dptr(pose_ligand, torch.int32), n, _dptr(genes, torch.float32), stride,
                                 _dptr(best_energy, torch.float32), _dptr(run_best, torch.float32),
                                 _dptr(n_evals, torch.int64), C.byref(prm), _stream(stream)))


def ad_lga_run(ctx, lig, n_runs, genes, energies, run_best=None, n_evals=None, n_gens=None, *, pop_size=150,
               max_gens=27000, max_evals=2_500_000, elitism=1, cross_rate=0.8, mut_rate=0.02, tour_rate=0.6,
               ls_rate=0.8, dmov=16.0, dang=90.0, seed=0, ls_iters=300, rho=0.8, eps=0.01, engine=AD_ENGINE_SIMT,
               warps_per_cta=0, stream=None) -> None:
    import torch
    n, stride = genes.shape
    assert n == n_runs * pop_size
    prm = LGAParams(pop_size, max_gens, max_evals, elitism, cross_rate, mut_rate, tour_rate, ls_rate, dmov, dang,
                    seed, LSParams(ls_iters, rho, eps, 0, engine, warps_per_cta, None, None))
    _check(lib().ad_lga_run(ctx, lig, n_runs, _dptr(genes, torch.float32), stride, _dptr(energies, torch.float32),
                            _dptr(run_best, torch.float32), _dptr(n_evals, torch.int64), _dptr(n_gens, torch.int32),
                            C.byref(prm), _stream(stream)))


def ad_reduce_blocks(ctx, engine, partials, out, stream=None) -> None:
    import torch
    nb, P, Cc = partials.shape
    _check(lib().ad_reduce_blocks(ctx, engine, nb, P, Cc, _dptr(partials, torch.float32), _dptr(out, torch.float32),
                                  _stream(stream)))


def ad_sync(ctx, stream=None) -> None:
    """Wait for the stream; raise AdError for device-side argument errors recorded so far."""
    _check(lib().ad_sync(ctx, _stream(stream)))


def ad_query(ctx, lig=-1):
    a, b, c = C.c_int32(), C.c_int32(), C.c_int32()
    _check(lib().ad_query(ctx, lig, C.byref(a), C.byref(b), C.byref(c)))
    return {"n_sms": a.value, "smem_per_pose": b.value, "blob_bytes": c.value}


def ad_last_launch(ctx):
    a, b, c = C.c_int32(), C.c_int32(), C.c_int32()
    _check(lib().ad_last_launch(ctx, C.byref(a), C.byref(b), C.byref(c)))
    out = {"grid": a.value, "block": b.value, "smem_bytes": c.value}
    try:  # inspection hook, not part of include/ad.h
        f = lib().adx_last_maxreg
        f.argtypes, f.restype = [C.c_void_p], C.c_int32
        out["maxreg"] = int(f(ctx))
    except AttributeError:
        pass
    return out


def pair_loop_kind(ctx, lig) -> int:
    """Inspection hook (not part of include/ad.h): 1 shared-memory cherries, 2 global-
    memory cherries, 0 other pair loops (which kernel twins a launch of it can use)."""
    try:
        f = lib().adx_pair_loop
    except AttributeError:
        return 0
    f.argtypes, f.restype = [C.c_void_p, C.c_int32], C.c_int32
    return int(f(ctx, lig))


# ---------------------------------------------------------------- convenience
class Context:
    """One device context: grids + ligands uploaded once, many score / LS calls."""

    def __init__(self, device: int = 0):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("libad needs a CUDA device (B200, sm_100a); there is no CPU fallback")
        self.device = device
        self.h = ad_context_create(device)
        self.ligs = {}

    def close(self):
        if self.h is not None:
            ad_context_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def upload_grid(self, grid):
        ad_upload_grids(self.h, grid)

    def upload_ligand(self, lig, ff) -> int:
        return ad_upload_ligand(self.h, lig, ff)

    def upload_ligands(self, ligs, ff, threads: int = 0) -> list:
        """Upload many ligands from a pool of host threads (ad_upload_ligand is
        thread-safe on one context and ctypes releases the GIL, so the host-side
        preparation of the pair schedules overlaps).  Returns the ids in order."""
        from concurrent.futures import ThreadPoolExecutor
        import os
        n = threads or max(1, min(len(ligs), len(os.sched_getaffinity(0))))
        with ThreadPoolExecutor(n) as ex:
            return list(ex.map(lambda L: ad_upload_ligand(self.h, L, ff), ligs))

    def sync(self) -> None:
        """ad_sync on the current stream: raises AdError for device-side errors."""
        ad_sync(self.h)

    def free_ligand(self, lig_id: int) -> None:
        ad_free_ligand(self.h, lig_id)

    def set_launch_ligands(self, ids=None) -> None:
        ad_set_launch_ligands(self.h, ids)

    def set_schedule_effort(self, effort: int) -> None:
        ad_set_schedule_effort(self.h, effort)

    def score(self, lig_id, genes, grad=True, aux=False, pose_ligand=None):
        import torch
        n, stride = genes.shape
        dev = genes.device
        E = torch.empty(n, dtype=torch.float32, device=dev)
        G = torch.zeros(n, stride, dtype=torch.float32, device=dev) if grad else None
        A = torch.empty(n, 8, dtype=torch.float32, device=dev) if aux else None
        ad_score_poses(self.h, lig_id, pose_ligand, genes, E, G, A)
        return E, G, A

    def local_search(self, lig_id, genes, *, max_iters=300, rho=0.8, eps=0.01, engine="simt", pop_per_run=0,
                     warps_per_cta=0, trace=False, pose_ligand=None, n_evals=None, phases=False):
        """In-place LS on `genes` (CUDA tensor [n, stride]); returns dict of outputs
        (phases=True: the A14 instrumented kernel, "phase_cycles" [n, 5] int64)."""
        import torch
        n, stride = genes.shape
        dev = genes.device
        bE = torch.empty(n, dtype=torch.float32, device=dev)
        rb = torch.empty(n // pop_per_run, 1 + stride, dtype=torch.float32, device=dev) if pop_per_run else None
        tr = torch.empty(n, max_iters, 1 + 2 * stride, dtype=torch.float32, device=dev) if trace else None
        ph = torch.zeros(n, 5, dtype=torch.int64, device=dev) if phases else None
        ad_local_search(self.h, lig_id, pose_ligand, genes, bE, rb, n_evals, max_iters=max_iters, rho=rho, eps=eps,
                        pop_per_run=pop_per_run, engine=ENGINES[engine] if isinstance(engine, str) else engine,
                        warps_per_cta=warps_per_cta, trace=tr, phase_cycles=ph)
        return {"best_energy": bE, "run_best": rb, "trace": tr, "phase_cycles": ph}

    def lga(self, lig_id, genes, n_runs, *, engine="simt", **kw):
        """NEXT-3 Lamarckian GA in place on `genes` (CUDA [n_runs * pop_size, stride])."""
        import torch
        n, stride = genes.shape
        dev = genes.device
        E = torch.empty(n, dtype=torch.float32, device=dev)
        rb = torch.empty(n_runs, 1 + stride, dtype=torch.float32, device=dev)
        ev = torch.empty(n_runs, dtype=torch.int64, device=dev)
        gn = torch.empty(n_runs, dtype=torch.int32, device=dev)
        ad_lga_run(self.h, lig_id, n_runs, genes, E, rb, ev, gn,
                   engine=ENGINES[engine] if isinstance(engine, str) else engine, **kw)
        return {"energies": E, "run_best": rb, "n_evals": ev, "n_gens": gn}
