"""Parity gates (reading Z18 of the north_star tolerance).

energy:   |E_gpu - E_oracle| <= 1e-3 + 2^-20 * (A_E + S_E)
gradient: ||g_gpu - g_oracle||_2 <= 1e-4 * max(||g_oracle||_2, 1e-2 * ||A_grad||_2)

A_E = sum over every energy term of |term| (inter corners weighted, vdW
attractive and repulsive parts separately); S_E = sum over terms of
|d term/d coordinates| x |coordinates| (the first-order effect of rounding the
atom coordinates, which FP32 carries with ~2^-24 relative error); A_grad = per
gene sum over terms of |Jacobian| . (|term gradient| + |d term gradient/dX| |X|).
All three come from the oracle (aux / agrad).  For sane poses A_E + S_E is a
few hundred, so the energy gate is the north_star's 1e-3 kcal/mol; for clashing
(r^-12) or out-of-grid poses FP32 cannot resolve 1e-3 of a 1e5 kcal/mol energy
and the gate scales with the magnitudes (16 FP32 ulps of them).
"""
import numpy as np


def energy_scale(aux):
    """A_E + S_E from the oracle's aux rows."""
    from oracle.oracle import AUX_ABS_E, AUX_SENS_E
    aux = np.asarray(aux)
    return aux[..., AUX_ABS_E] + aux[..., AUX_SENS_E]


def energy_gate(E_gpu, E_ora, scale):
    E_gpu = np.asarray(E_gpu, np.float64)
    return np.abs(E_gpu - E_ora) <= 1e-3 + 2.0 ** -20 * np.asarray(scale)


def grad_gate(g_gpu, g_ora, agrad):
    g_gpu = np.asarray(g_gpu, np.float64)
    d = np.linalg.norm(g_gpu - g_ora, axis=-1)
    scale = np.maximum(np.linalg.norm(g_ora, axis=-1), 1e-2 * np.linalg.norm(agrad, axis=-1))
    return d <= 1e-4 * scale


def rel_grad_err(g_gpu, g_ora, agrad):
    g_gpu = np.asarray(g_gpu, np.float64)
    d = np.linalg.norm(g_gpu - g_ora, axis=-1)
    scale = np.maximum(np.linalg.norm(g_ora, axis=-1), 1e-2 * np.linalg.norm(agrad, axis=-1))
    return d / np.maximum(scale, 1e-300)
