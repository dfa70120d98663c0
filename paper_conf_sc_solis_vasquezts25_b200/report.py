"""Measurement helpers: the paper's Amdahl model and the algorithmic work model.

amdahl_speedup: Eq 6, predicted T_baseline / T_TCEC = 1 / (f/S + (1 - f)),
with f = f_eff and S = TC / SIMT peak ratio.
"""
from __future__ import annotations


def amdahl_speedup(f: float, S: float) -> float:
    return 1.0 / (f / S + (1.0 - f))


def work_per_eval(n_atoms: int, n_tors: int, n_pairs: int, l_rot: int, m_sum: int) -> dict:
    """Algorithmic work of one energy+gradient evaluation (SURVEY §8(d) model, FMA = 2 flops):
        F    = 24 T + 30 L_rot + 200 N + 75 P + 19 N + 17 M_sum + 15 G
        MUFU = 5 P + N + T + 2 G
        L2   = 96 N bytes (3 maps x 8 corners x 4 B gathered per atom)
    L_rot = sum over atoms of (1 + torsions moving the atom); M_sum = sum_b |M_b|."""
    G = 6 + n_tors
    flops = 24 * n_tors + 30 * l_rot + 200 * n_atoms + 75 * n_pairs + 19 * n_atoms + 17 * m_sum + 15 * G
    mufu = 5 * n_pairs + n_atoms + n_tors + 2 * G
    return {"flops": float(flops), "mufu": float(mufu), "l2_bytes": float(96 * n_atoms)}


def ligand_work(lig) -> dict:
    """work_per_eval for a synth.Ligand."""
    m_sum = int(lig.tors_moving.sum()) if lig.n_tors else 0
    l_rot = lig.n_atoms + m_sum
    return work_per_eval(lig.n_atoms, lig.n_tors, lig.n_pairs, l_rot, m_sum)


# B200 FP32 SIMT peak from unit counts and clock: 148 SMs x 128 FP32
# lanes x 2 flops (FMA) x f_clk.  At the 1965 MHz max clock: 74.4 TFLOP/s.
B200_SMS = 148
B200_FP32_LANES_PER_SM = 128
B200_MUFU_PER_SM_PER_CLK = 16


def fp32_peak_tflops(sm_mhz: float) -> float:
    return B200_SMS * B200_FP32_LANES_PER_SM * 2 * sm_mhz * 1e6 / 1e12
