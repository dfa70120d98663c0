#!/usr/bin/env python
"""Benchmark: pose energy+gradient evaluations per second of the ADADELTA local
search (BASELINE.json metric) on the drug-like workload (config 2: 40 atoms,
8 torsions, 60^3 grid, 20 runs x 150 pop x 300 iterations = 9.0e5 evals per
GPU per step), plus max |dE| vs the FP64 oracle.

One step = one whole hot-path pass: restore the start genotypes (D2D), one
ad_local_search call (ADADELTA kernel + best-of-run kernel), and for N > 1 the
NCCL all_gather of the best-pose records.  Weak scaling: every rank runs its own
config-2 replica (seed = 2000 + rank).  L2 is flushed (256 MiB write) between
timed steps, outside the timed events.

Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--engine simt|tc|paper]
       python bench.py --impl reference ...   (times the FP64 oracle on host cores)
Under torchrun (N > 1) every rank runs; rank 0 prints ONE JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "pose energy+gradient evals/sec (1/2/4/8 B200); max |ΔE| vs FP64 oracle"
UNIT = "evals/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    # default = the faster engine measured on this workload (the TC engine is kept
    # only if it wins, north_star); `--engine tc` times the tensor-core engine
    ap.add_argument("--engine", default="simt", choices=["simt", "tc", "tc_fp16", "paper", "paper_tcec"])
    ap.add_argument("--warps", type=int, default=0, help="warps per CTA (0 = library choice)")
    ap.add_argument("--config", type=int, default=2, choices=[2, 3, 5])
    # config 5 (virtual screen, strong scaling over the ranks)
    ap.add_argument("--ligands", type=int, default=8192, help="config 5: ligands in the screen")
    ap.add_argument("--effort", type=int, default=1, help="config 5: pair-schedule placement effort (0..2)")
    ap.add_argument("--buckets", type=int, default=8, help="config 5: launches per rank per step")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-paper-engine", action="store_true")
    ap.add_argument("--no-lga", action="store_true", help="skip the full LGA docking-job measurement")
    return ap.parse_args()


def workload_config(w, lig, engine, extra=None):
    c = {
        "workload": f"{w.name}: {lig.n_atoms} atoms, {lig.n_tors} torsions, {lig.n_pairs} intra pairs, "
                    f"{w.grid.nx}^3 grid x {w.grid.spacing} A ({w.grid.n_maps} maps), {w.runs} runs x {w.pop} pop "
                    f"x {w.iters} ADADELTA iterations per GPU",
        "poses": w.n_poses, "iters": w.iters, "runs": w.runs, "pop": w.pop,
        "engine": engine, "l2": "flushed between timed steps (256 MiB write, outside the timed events)",
        "inputs": "seeded synthetic ligand/receptor grids (paper_conf_sc_solis_vasquezts25_b200/synth.py)",
    }
    if extra:
        c.update(extra)
    return c


class ClockSampler:
    """SM clock + throttle reasons polled every 2 ms through NVML during the timed
    region (the timed region of a default run is only tens of ms); falls back to
    `nvidia-smi -lms 200` if NVML is unavailable."""

    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.sm, self.max_sm, self.reasons = [], None, set()
        self._stop = threading.Event()
        self.proc = None

    def __enter__(self):
        try:
            import pynvml as N
            N.nvmlInit()
            visible = os.environ.get("CUDA_VISIBLE_DEVICES")
            phys = int(visible.split(",")[self.idx]) if visible else self.idx
            h = N.nvmlDeviceGetHandleByIndex(phys)
            self.max_sm = float(N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM))
            get_r = getattr(N, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                N.nvmlDeviceGetCurrentClocksThrottleReasons

            def sample():
                self.sm.append(float(N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)))
                r = int(get_r(h))
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)

            def poll():
                while not self._stop.wait(0.002):
                    sample()
            self._sample = sample
            self._switch = sys.getswitchinterval()
            sys.setswitchinterval(0.0005)  # let the poller in while the main thread launches
            self.th = threading.Thread(target=poll, daemon=True)
            self.th.start()
            self.mode = "nvml 2 ms"
        except Exception:  # noqa: BLE001
            q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
            self.mode = "nvidia-smi 200 ms"
            try:
                self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={q}",
                                              "--format=csv,noheader,nounits", "-lms", "200"],
                                             stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
                self.th = threading.Thread(target=self._read, daemon=True)
                self.th.start()
            except FileNotFoundError:
                self.proc = None
        return self

    def _read(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            try:
                self.sm.append(float(parts[0]))
                self.max_sm = float(parts[1])
            except (ValueError, IndexError):
                continue
            for n, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    self.reasons.add(n)

    def __exit__(self, *a):
        if hasattr(self, "_sample"):
            self._sample()  # at least one sample at the end of the timed region
            sys.setswitchinterval(self._switch)
        self._stop.set()
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        elif hasattr(self, "th"):
            self.th.join(timeout=1)

    def summary(self):
        return {"sm_mhz": statistics.median(self.sm) if self.sm else None, "sm_max_mhz": self.max_sm,
                "reasons": sorted(self.reasons), "samples": len(self.sm), "sampler": getattr(self, "mode", None)}


def load_co_bounds(engine, config):
    """Issue and L1/shared data-pipe utilisation of the LS kernel from the committed
    ncu --set full summary of the same workload (profiles/ncu_summary.json), if any."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        k = json.load(open(path)).get("ls_kernel", {}).get(f"config{config}_{engine}")
        if not k or "issue_active_pct" not in k:
            return None
        return {"issue_active": k["issue_active_pct"] / 100.0, "l1tex_throughput": k["l1tex_throughput_pct"] / 100.0,
                "tensor_pipe_frac": k.get("tensor_pipe_pct", 0.0) / 100.0,
                "warp_instructions_per_launch": k.get("warp_instructions"),
                "shared_wavefronts_per_launch": k.get("shared_wavefronts"),
                "source": f"profiles/ncu_{k['round']}.md ({k['report']}, ncu --set full)"}
    except (OSError, ValueError, KeyError):
        return None


def load_traffic(engine, config):
    """dram bytes per launch of the LS kernel from a committed ncu --set full summary, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(path))
        k = d.get("ls_kernel", {}).get(f"config{config}_{engine}")
        return None if k is None else float(k["dram_bytes_per_launch"])
    except (OSError, ValueError, KeyError):
        return None


def parity_report(O, ctx, lid, w, start, genes, cores, ns=512):
    """max |dE| and gradient error vs the FP64 oracle (gates of tests/parity.py,
    DESIGN.md "Tolerances"): the first `ns` start poses and the `ns` relaxed poses
    (best genotypes) the timed launches returned, both through ad_score_poses in
    the bench launch configuration.  sane = A_E < 500: there the plain north_star
    numbers (|dE| <= 1e-3, ||dg|| / ||g|| <= 1e-4) are reported as they are."""
    import torch
    from tests import parity as P
    lig = w.ligands[0]
    Gn = lig.n_genes
    out = {"gate": "Z18: |dE| <= 1e-3 + 2^-20 A_E (sane, A_E < 500), clash gate 1e-3 + 2^-20 (A_E + S_E) "
                   "(A_E >= 500); ||dg|| <= 1e-4 max(||g||, 1e-2 ||A_grad||) (DESIGN.md Tolerances)"}
    for kind, g in (("start_poses", start[:ns]), ("relaxed_poses", genes[:ns])):
        g = g.contiguous()
        Eg, Gg, _ = ctx.score(lid, g, grad=True)
        torch.cuda.synchronize()
        Eg, Gg = Eg.cpu().numpy(), Gg.cpu().numpy()[:, :Gn]
        Eo, Go, aux, ag = O.score(lig, w.grid, w.ff, g.cpu().numpy(), threads=cores)
        Go, ag = Go[:, :Gn], ag[:, :Gn]
        dE = np.abs(Eg.astype(np.float64) - Eo)
        rel = P.rel_grad_err(Gg, Go)
        sane = P.sane(aux)
        kink = aux[:, O.AUX_MARGIN_G] < 1e-4
        r = {"n": int(ns), "n_sane_poses": int(sane.sum()), "max_abs_dE": float(dE.max()),
             "median_abs_dE": float(np.median(dE)),
             "frac_within_gates": float(np.mean(P.energy_gate(Eg, Eo, aux) & (P.grad_gate(Gg, Go, ag) | kink))),
             "max_grad_err_over_z18_scale": float(P.rel_grad_err(Gg, Go, ag).max()),
             "n_kink_poses": int(kink.sum())}
        if sane.any():
            r.update({"sane_max_abs_dE": float(dE[sane].max()),
                      "sane_frac_abs_dE_le_1e-3": float(np.mean(dE[sane] <= 1e-3)),
                      "sane_max_grad_rel_err": float(rel[sane].max()),
                      "sane_max_grad_rel_err_no_kink": float(rel[sane & ~kink].max()) if (sane & ~kink).any() else None,
                      "sane_median_grad_rel_err": float(np.median(rel[sane])),
                      "sane_frac_grad_rel_err_le_1e-4": float(np.mean(rel[sane] <= 1e-4))})
        r["sample"] = (f"first {ns} start poses of {w.name}" if kind == "start_poses" else
                       f"best genotypes of the first {ns} poses after the timed LS launches")
        out[kind] = r
    return out


def paper_engines(ad, ctx, lid, w, start, bestE, flush, stream, ours_ms, block_sizes=(64, 128, 256)):
    """The paper-style kernel (one block per pose) at the paper's block sizes
    (Fig 4, Tab 5): SIMT baseline (7 sequential block
    reductions) and TCEC (one error-corrected TF32 tensor-core reduction,
    P:L186-199), median of 3 L2-flushed launches each, plus the A14 reduction
    fraction f of each (instrumented twin, one launch).  The headline speedup is
    over the FASTEST paper-style baseline."""
    import torch

    def time_engine(eng, threads):
        gp = start.clone()
        ad.ad_local_search(ctx.h, lid, None, gp, bestE, None, None, max_iters=w.iters, engine=eng,
                           warps_per_cta=threads)
        ts = []
        for k in range(3):
            gp.copy_(start)
            flush.fill_(float(k))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            ad.ad_local_search(ctx.h, lid, None, gp, bestE, None, None, max_iters=w.iters, engine=eng,
                               warps_per_cta=threads)
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return statistics.median(ts)

    def reduction_fraction(eng, threads):
        gp = start.clone()
        out = ctx.local_search(lid, gp, max_iters=w.iters, engine=eng, warps_per_cta=threads, phases=True)
        torch.cuda.synchronize()
        ph = out["phase_cycles"].double().sum(0).cpu().numpy()
        return float(ph[3] / ph.sum())

    rows = {}
    for t in block_sizes:
        r = {}
        for name, eng in (("baseline", ad.AD_ENGINE_PAPER_BASELINE), ("tcec", ad.AD_ENGINE_PAPER_TCEC)):
            r[f"{name}_ms"] = time_engine(eng, t)
            r[f"{name}_f"] = reduction_fraction(eng, t)
        r["tcec_over_baseline"] = r["baseline_ms"] / r["tcec_ms"]
        rows[str(t)] = r
    best_t = min(rows, key=lambda t: rows[t]["baseline_ms"])
    best = rows[best_t]["baseline_ms"]
    return {"engine": "paper-style kernel (self-built: this build's pose / inter / intra code, one block per pose, "
                      "P:L128): 7 sequential block reductions (SIMT baseline, P:L132) or one error-corrected TF32 "
                      "tensor-core reduction (TCEC, P:L186-199)",
            "by_block_size": rows, "fastest_baseline_block": int(best_t), "fastest_baseline_ms": best,
            "fastest_baseline_evals_per_s": w.n_poses * w.iters / (best / 1e3),
            "speedup_of_this_engine_over_fastest_baseline": best / ours_ms,
            "denominator": "self-built paper-style kernel (no reference implementation is available)",
            "paper_target_speedup": 1.35,
            "paper_reported": "B200 TCEC/baseline 1.35x (42 cases, 256 threads, P:L299/L383); 1.45x 7cpa 128 threads "
                              "(Tab 5 P:L344)"}


def run_reference_screen(args, O, synth):
    """--impl reference --config 5: the oracle on a bounded sample of the screen
    (every step: 1 run x pop poses x 300 iterations of 8 ligands spread over the
    size draws), evals/s on the host cores."""
    spec = synth.ScreenSpec(n_ligands=args.ligands)
    cores = len(os.sched_getaffinity(0))
    ff = synth.FFParams()
    ks = sorted(range(spec.n_ligands), key=lambda k: spec.sizes[k])
    ks = [ks[int(i)] for i in np.linspace(0, len(ks) - 1, 8)]
    work = [(spec.ligand(k), spec.genes(k)[:spec.pop]) for k in ks]
    for _ in range(args.warmup):
        O.local_search(work[0][0], spec.grid, ff, work[0][1], max_iters=spec.iters, threads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        for L, g in work:
            O.local_search(L, spec.grid, ff, g, max_iters=spec.iters, threads=cores)
    dt = time.perf_counter() - t0
    val = args.steps * len(work) * spec.pop * spec.iters / dt
    sample = (f"1 run x {spec.pop} pop x {spec.iters} ADADELTA iterations of 8 of the {spec.n_ligands} screen "
              f"ligands ({work[0][0].n_atoms}-{work[-1][0].n_atoms} atoms) per step")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{spec.name}: {spec.n_ligands} ligands x {spec.runs} runs x {spec.pop} pop x "
                               f"{spec.iters} ADADELTA iterations", "engine": "oracle", "sample": sample},
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}), flush=True)


def run_reference(args):
    """--impl reference: the FP64 oracle as it stands, on host cores, rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import oracle as O
    from paper_conf_sc_solis_vasquezts25_b200 import synth
    if args.config == 5:
        run_reference_screen(args, O, synth)
        return
    w = synth.make_config(args.config)
    lig = w.ligands[0]
    cores = len(os.sched_getaffinity(0))
    n_sample = 8 * cores if args.config == 2 else 2 * cores
    genes = w.genes[:n_sample]
    for _ in range(args.warmup):
        O.local_search(lig, w.grid, w.ff, genes[:cores], max_iters=w.iters, threads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        O.local_search(lig, w.grid, w.ff, genes, max_iters=w.iters, threads=cores)
    dt = time.perf_counter() - t0
    evals = args.steps * n_sample * w.iters
    val = evals / dt
    sample = f"{n_sample} poses x {w.iters} ADADELTA iterations of {w.name} per step (of {w.n_poses} poses)"
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(w, lig, "oracle", {"sample": sample}),
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_screen_bench(args):
    """Config 5: the virtual screen (8192 ligands of 20-110 atoms and 0-32 torsions
    x 20 runs x 16 pop x 300 ADADELTA iterations against the config-2 receptor),
    (ligand, run) units LPT-sharded over the ranks, one NCCL all_gather of the
    best-pose records per step.  Strong scaling: the total work is fixed.  One
    step = every bucket launch of the rank + the gather; ligands are uploaded
    (and their pair schedules built) once, before the timed region, like the
    receptor grids."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_solis_vasquezts25_b200 import ad, dist as addist, report, screen, synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    if world > 1:
        torch.cuda.set_device(local)
        addist.init_process_group("nccl", torch.device("cuda", local))
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    cores = len(os.sched_getaffinity(0))
    spec = synth.ScreenSpec(n_ligands=args.ligands)
    ff = synth.FFParams()
    ctx = ad.Context(local)
    S = screen.Screen(ctx, spec, ff, rank=rank, world=world, engine=args.engine, n_buckets=args.buckets,
                      effort=args.effort, upload_threads=max(1, cores // local_world),
                      gen_processes=max(1, cores // local_world))
    stream = torch.cuda.current_stream()
    n_evals = torch.zeros(1, dtype=torch.int64, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    for _ in range(args.warmup):
        S.step()
    torch.cuda.synchronize()
    n_evals.zero_()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with ClockSampler(local) as clocks:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        for k in range(args.steps):
            flush.fill_(float(k))  # L2 flush, outside the timed events
            ev[k][0].record(stream)
            rec = S.step(n_evals)
            ev[k][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    ms = [a.elapsed_time(b) for a, b in ev]
    total = torch.tensor([sum(ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(total, op=dist.ReduceOp.MAX)
    total_ms = float(total.item())
    assert int(n_evals.item()) == args.steps * S.n_poses * spec.iters
    evals_all = args.steps * spec.n_ligands * spec.runs * spec.pop * spec.iters
    value = evals_all / (total_ms / 1e3)
    recs = rec.cpu().numpy()
    got = recs[~np.isnan(recs[:, 0])]
    assert len(got) == spec.n_ligands * spec.runs and np.all(np.isfinite(got[:, 2])), "screen records incomplete"

    # end to end: the start genotypes from pinned host memory + the records back, per step
    h2d = S.pin_host_inputs()
    h_rec = torch.empty(tuple(rec.shape)).pin_memory()
    e2e = []
    for k in range(max(2, args.steps)):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        flush.fill_(float(k))
        a.record(stream)
        r = S.step(from_host=True)
        h_rec.copy_(r, non_blocking=True)
        b.record(stream)
        e2e.append((a, b))
    torch.cuda.synchronize()
    e2e_t = torch.tensor([sum(a.elapsed_time(b) for a, b in e2e) / len(e2e)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_val = spec.n_ligands * spec.runs * spec.pop * spec.iters / (float(e2e_t.item()) / 1e3)

    # roofline of this rank's LS launches: the flop model per ligand x its evaluations
    flops = sum(report.ligand_work(S.ligands[k])["flops"] for b in S.buckets for k, _ in b["units"]) * spec.pop * spec.iters
    achieved = flops / (statistics.mean(ms) / 1e3) / 1e12
    peak = report.fp32_peak_tflops(1965.0)
    roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": None, "peak_basis": "148 SMs x 128 FP32 lanes x 2 (FMA) x 1965 MHz max SM clock (DESIGN.md)",
                "flops_per_step_rank0": flops, "launches_per_step": len(S.buckets)}

    cpu = parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import oracle as O
        from tests import parity as P
        # the oracle on a bounded sample: the first 2 runs (32 poses, 300 iterations) of 12
        # ligands spread over the size range; and the GPU's best energies of those units
        # re-scored by the oracle at the returned genotypes
        ks = sorted(S.ligands, key=lambda k: S.ligands[k].n_pairs)
        ks = [ks[int(i)] for i in np.linspace(0, len(ks) - 1, 12)]
        t0 = time.perf_counter()
        n_s = 0
        for k in ks:
            g = spec.genes(k)[:2 * spec.pop]
            O.local_search(S.ligands[k], spec.grid, ff, g, max_iters=spec.iters, threads=cores)
            n_s += len(g) * spec.iters
        dt = time.perf_counter() - t0
        cpu = {"value": n_s / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"2 runs x {spec.pop} pop x {spec.iters} ADADELTA iterations of 12 screen ligands "
                         f"({S.ligands[ks[0]].n_atoms}-{S.ligands[ks[-1]].n_atoms} atoms)"}
        by_unit = {(int(r[0]), int(r[1])): r for r in got}
        dE, ok = [], []
        for k in ks:
            L = S.ligands[k]
            for r in range(spec.runs):
                row = by_unit[(k, r)]
                Eo, _, aux, _ = O.score(L, spec.grid, ff, row[3:3 + spec.stride][None, :].astype(np.float32))
                d = abs(float(row[2]) - float(Eo[0]))
                dE.append(d)
                ok.append(bool(P.energy_gate(np.float32(row[2])[None], Eo, aux)[0]))
        parity = {"max_abs_dE": float(max(dE)), "median_abs_dE": float(np.median(dE)),
                  "frac_within_gate": float(np.mean(ok)),
                  "gate": "Z18 |dE| <= 1e-3 + 2^-20 A_E (A_E < 500), clash gate 2^-20 (A_E + S_E) above "
                          "(DESIGN.md Tolerances)",
                  "sample": f"best pose of every run of 12 ligands ({len(dE)} records) re-scored by the FP64 oracle"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{spec.name}: {spec.n_ligands} ligands (20-110 atoms, 0-32 torsions) x "
                                   f"{spec.runs} runs x {spec.pop} pop x {spec.iters} ADADELTA iterations, 60^3 grid "
                                   f"x 0.375 A (10 maps), (ligand, run) units LPT-sharded over {world} GPU(s)",
                       "engine": args.engine, "buckets_per_rank": len(S.buckets), "schedule_effort": args.effort,
                       "l2": "flushed between timed steps (256 MiB write, outside the timed events)",
                       "parallelism": f"units sharded, {world} GPU(s), NCCL all_gather of best-pose records",
                       "setup_s_rank0": S.setup_s},
            "roofline": roofline, "cpu_baseline": cpu, "parity": parity,
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(h_rec.numel() * 4)},
            "clocks": clocks.summary(), "gpu_launches": 2 * len(S.buckets) * args.steps,  # LS + best-of-run
        }
        print(json.dumps(line), flush=True)
    S.close()
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    if args.config == 5:
        run_screen_bench(args)
        return
    import torch
    import torch.distributed as dist

    from paper_conf_sc_solis_vasquezts25_b200 import ad, dist as addist, report, synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        torch.cuda.set_device(local)
        addist.init_process_group("nccl", torch.device("cuda", local))
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)

    # config 2: weak scaling (every rank its own replica, seed 2000 + rank); config 3:
    # strong scaling (the 100 runs of replica 0 LPT-sharded over the ranks)
    strong = args.config == 3
    w = synth.make_config(args.config, replica=0 if strong else rank)
    lig = w.ligands[0]
    stride = lig.n_genes
    shards = addist.lpt_shard([1.0] * w.runs, world) if strong else None
    my_runs = shards[rank] if strong else list(range(w.runs))
    n_runs = len(my_runs)
    my_genes = np.ascontiguousarray(np.concatenate([w.genes[r * w.pop:(r + 1) * w.pop] for r in my_runs]))
    ctx = ad.Context(local)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(lig, w.ff)
    start = torch.from_numpy(my_genes).to(dev)
    genes = start.clone()
    n = n_runs * w.pop
    bestE = torch.empty(n, device=dev)
    run_best = torch.empty(max(len(s) for s in shards) if strong else w.runs, 1 + stride, device=dev)
    n_evals = torch.zeros(1, dtype=torch.int64, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()
    engine = ad.ENGINES[args.engine]
    wpc = args.warps if not args.engine.startswith("paper") else (args.warps or 64)

    def step(ev=None):
        genes.copy_(start)
        if ev:
            ev[0].record(stream)
        ad.ad_local_search(ctx.h, lid, None, genes, bestE, run_best[:n_runs], n_evals, max_iters=w.iters,
                           pop_per_run=w.pop, engine=engine, warps_per_cta=wpc)
        if ev:
            ev[1].record(stream)
        if world > 1:
            addist.gather_records(run_best)

    nvtx = torch.cuda.nvtx  # ranges on the Nsight timeline; libad adds one per ABI call
    with nvtx.range("bench.warmup"):
        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ev_step = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    ev_kern = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    n_evals.zero_()
    with ClockSampler(local) as clocks, nvtx.range("bench.timed"):
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        for k in range(args.steps):
            flush.fill_(float(k))  # L2 flush, outside the timed events
            ev_step[k][0].record(stream)
            step(ev_kern[k])
            ev_step[k][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev_step]
    kern_ms = [a.elapsed_time(b) for a, b in ev_kern]
    launch = ad.ad_last_launch(ctx.h)
    total = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(total, op=dist.ReduceOp.MAX)
    total_ms = float(total.item())
    assert int(n_evals.item()) == args.steps * n * w.iters
    evals_all = args.steps * w.iters * (w.n_poses if strong else world * n)
    value = evals_all / (total_ms / 1e3)

    # ---- end to end through the public API with HOST buffers (pinned) ----
    h_genes = torch.from_numpy(my_genes).pin_memory()
    h_bestE = torch.empty(n).pin_memory()
    h_run = torch.empty(n_runs, 1 + stride).pin_memory()
    e2e_ev = []
    nvtx.range_push("bench.e2e")
    for k in range(max(2, args.steps)):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        flush.fill_(float(k))
        a.record(stream)
        genes.copy_(h_genes, non_blocking=True)
        ad.ad_local_search(ctx.h, lid, None, genes, bestE, run_best[:n_runs], None, max_iters=w.iters,
                           pop_per_run=w.pop, engine=engine, warps_per_cta=wpc)
        h_bestE.copy_(bestE, non_blocking=True)
        h_run.copy_(run_best[:n_runs], non_blocking=True)
        b.record(stream)
        e2e_ev.append((a, b))
    torch.cuda.synchronize()
    nvtx.range_pop()
    e2e_ms = sum(a.elapsed_time(b) for a, b in e2e_ev) / len(e2e_ev)
    e2e_t = torch.tensor([e2e_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_val = (w.n_poses if strong else world * n) * w.iters / (float(e2e_t.item()) / 1e3)

    # ---- config 1 (BASELINE configs[0]): ONE ad_score_poses call (256 poses, energy + gradient)
    # end to end with host buffers -- pinned H2D of the genotypes, the call, D2H of energies and
    # gradients, synchronize -- timed on the host clock per call (the latency a GA driver sees) ----
    call1 = None
    if rank == 0:
        w1 = synth.make_config(1)
        ctx1 = ad.Context(local)
        try:
            ctx1.upload_grid(w1.grid)
            lid1 = ctx1.upload_ligand(w1.ligands[0], w1.ff)
            hg1 = torch.from_numpy(np.ascontiguousarray(w1.genes)).pin_memory()
            g1 = torch.empty_like(hg1, device=dev)
            n1, s1 = hg1.shape
            out1 = torch.empty(n1 * (1 + s1), device=dev)  # energies then gradients: ONE D2H copy
            E1, G1 = out1[:n1], out1[n1:].view(n1, s1)
            hout1 = torch.empty(n1 * (1 + s1)).pin_memory()
            host_us, dev_us = [], []
            for k in range(230):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                a.record(stream)
                g1.copy_(hg1, non_blocking=True)
                ad.ad_score_poses(ctx1.h, lid1, None, g1, E1, G1)
                hout1.copy_(out1, non_blocking=True)
                b.record(stream)
                b.synchronize()
                t1 = time.perf_counter()
                if k >= 30:
                    host_us.append((t1 - t0) * 1e6)
                    dev_us.append(a.elapsed_time(b) * 1e3)
            call1 = {"workload": f"{w1.name}: {w1.n_poses} poses, energy + gene gradient, one ad_score_poses call",
                     "us_per_call_host_median": statistics.median(host_us),
                     "us_per_call_device_median": statistics.median(dev_us),
                     "evals_per_s_e2e": w1.n_poses / (statistics.median(host_us) / 1e6),
                     "h2d_bytes": int(hg1.numel() * 4), "d2h_bytes": int(hout1.numel() * 4),
                     "calls": len(host_us)}
        finally:
            ctx1.close()

    # ---- NEXT-3: the whole Lamarckian GA docking job on this workload (Alg 1) with the
    # paper's budgets (2.5e6 evaluations / 27 000 generations per run) -- the end-to-end
    # number the paper quotes as us per evaluation (A100, real ligand: context only) ----
    lga = None
    if rank == 0 and not args.no_lga and not args.engine.startswith("paper"):
        g_lga = start.clone()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        out = ctx.lga(lid, g_lga, n_runs, engine=args.engine, pop_size=w.pop, max_evals=2_500_000, max_gens=27000,
                      ls_iters=w.iters, seed=1)
        b.record(stream)
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        ev = int(out["n_evals"].sum().item())
        lga = {"runs": n_runs, "pop": w.pop, "budget": "2.5e6 evaluations or 27 000 generations per run (P:L57)",
               "evaluations": ev, "generations_max": int(out["n_gens"].max().item()), "seconds": ms / 1e3,
               "evals_per_s": ev / (ms / 1e3), "us_per_eval": ms * 1e3 / ev,
               "best_energy_median": float(out["run_best"][:, 0].median().item())}

    # ---- paper-style block-per-pose engines, same workload (the self-built speedup denominator) ----
    paper = None
    if rank == 0 and not args.no_paper_engine and not args.engine.startswith("paper"):
        paper = paper_engines(ad, ctx, lid, w, start, bestE, flush, stream, statistics.median(kern_ms))

    # ---- roofline of the dominant kernel (LS kernel), FP32 ALU bound ----
    work = report.ligand_work(lig)
    kern_avg_s = statistics.mean(kern_ms) / 1e3
    achieved = work["flops"] * n * w.iters / kern_avg_s / 1e12
    ck = clocks.summary()
    peak = report.fp32_peak_tflops(1965.0)
    roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": load_traffic(args.engine, args.config),
                "peak_basis": "148 SMs x 128 FP32 lanes x 2 (FMA) x 1965 MHz max SM clock (DESIGN.md)",
                "flops_per_eval": work["flops"], "mufu_per_eval": work["mufu"],
                "mufu_frac": work["mufu"] * n * w.iters / kern_avg_s / (148 * 16 * 1965e6),
                "l2_gather_gbs": work["l2_bytes"] * n * w.iters / kern_avg_s / 1e9,
                "kernel_ms_avg": kern_avg_s * 1e3,
                # north_star asks for HBM GB/s too: the ncu-measured DRAM bytes of one LS launch
                # (first touch of the maps; they stay L2-resident) over the live kernel time
                "hbm_gbs": (load_traffic(args.engine, args.config) or 0.0) / kern_avg_s / 1e9,
                # the units that actually bound the kernel: the FP32 flop model
                # counts useful arithmetic only, issue slots and the L1/shared pipe saturate first
                "co_bounds": load_co_bounds(args.engine, args.config)}

    # ---- CPU baseline (the oracle as it stands) + max |dE| vs the oracle ----
    cpu = None
    max_dE = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import oracle as O
        cores = len(os.sched_getaffinity(0))
        # a bounded sample of ~20 core-seconds of oracle work: chunks of 2 poses per core
        # (300 iterations each) until the budget is spent or the workload is exhausted
        budget_s = max(1.0, 20.0 / cores)
        n_s, chunk, dt = 0, 2 * cores, 0.0
        while n_s < w.n_poses and dt < budget_s:
            m = min(chunk, w.n_poses - n_s)
            t0 = time.perf_counter()
            O.local_search(lig, w.grid, w.ff, w.genes[n_s:n_s + m], max_iters=w.iters, threads=cores)
            dt += time.perf_counter() - t0
            n_s += m
        cpu = {"value": n_s * w.iters / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"{n_s} of the {w.n_poses} poses x {w.iters} ADADELTA iterations of {w.name} "
                         f"({dt:.1f} s on {cores} threads)"}
        max_dE = parity_report(O, ctx, lid, w, start, genes, cores)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": workload_config(w, lig, args.engine, {"parallelism": (
                                          f"the {w.runs} runs LPT-sharded over {world} GPU(s) (strong scaling), NCCL "
                                          "all_gather of the best-pose records" if strong else
                                          f"one replica per GPU ({world} GPU(s), weak scaling), NCCL all_gather of "
                                          "the best-pose records"),
                                                            "runs_this_rank": n_runs,
                                                            "launch": launch,
                                                            "intra_mode": os.environ.get("AD_INTRA_MODE", "scatter")}),
            "roofline": roofline, "cpu_baseline": cpu, "parity": max_dE,
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": int(h_genes.numel() * 4),
                    "d2h_bytes_per_step": int((h_bestE.numel() + h_run.numel()) * 4)},
            "clocks": ck, "gpu_launches": 2 * args.steps,
            "config1_score_call": call1,
            "lga": lga,
            "paper_baseline_engine": paper,
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
