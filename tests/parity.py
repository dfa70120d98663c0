"""Parity gates: reading Z18 of the north_star tolerance (SURVEY.md §8(c) Z18,
DESIGN.md "Tolerances").

Z18 energy gate   |E_gpu - E_oracle| <= 1e-3 + 2^-20 A_E
Z18 gradient gate ||g_gpu - g_oracle||_2 <= 1e-4 max(||g_oracle||_2, 1e-2 ||A_grad||_2)

A_E    = sum over every energy term of |term|              (oracle aux[AUX_ABS_E])
A_grad = per gene, sum of |summand| of the O-4 chain rule  (oracle agrad)
         dE/dg_k = sum_i dX_i/dg_k . g_i with g_i split into its terms.

A pose is SANE when A_E < 500 (Z18: there the energy gate is the north_star's
1e-3 kcal/mol up to 2^-20 A_E < 5e-4).  Clashing poses (A_E >= 500: r^-12
contacts, atoms out of the grid) cannot be resolved to 2^-20 A_E in FP32,
because rounding the atom coordinates alone moves a 1e5 kcal/mol wall energy
by more; they are held to a separately labelled CLASH gate that adds S_E, the
first-order effect of coordinate rounding (oracle aux[AUX_SENS_E]):

clash energy gate |dE| <= 1e-3 + 2^-20 (A_E + S_E)      (A_E >= 500 only)

The gradient gate is the Z18 gate for every pose.
"""
import numpy as np

SANE_AE = 500.0


def _aux(aux, name):
    from oracle import oracle as O
    return np.asarray(aux)[..., getattr(O, name)]


def sane(aux):
    """A_E < 500: poses the plain Z18 energy gate applies to."""
    return _aux(aux, "AUX_ABS_E") < SANE_AE


def z18_energy_tol(aux):
    return 1e-3 + 2.0 ** -20 * _aux(aux, "AUX_ABS_E")


def clash_energy_tol(aux):
    return 1e-3 + 2.0 ** -20 * (_aux(aux, "AUX_ABS_E") + _aux(aux, "AUX_SENS_E"))


def energy_tol(aux):
    """Per pose: the Z18 gate on sane poses, the labelled clash gate on the others."""
    return np.where(sane(aux), z18_energy_tol(aux), clash_energy_tol(aux))


def energy_gate(E_gpu, E_ora, aux):
    E_gpu = np.asarray(E_gpu, np.float64)
    return np.abs(E_gpu - E_ora) <= energy_tol(aux)


def grad_scale(g_ora, agrad):
    return np.maximum(np.linalg.norm(g_ora, axis=-1), 1e-2 * np.linalg.norm(agrad, axis=-1))


def grad_gate(g_gpu, g_ora, agrad):
    g_gpu = np.asarray(g_gpu, np.float64)
    d = np.linalg.norm(g_gpu - g_ora, axis=-1)
    return d <= 1e-4 * grad_scale(g_ora, agrad)


def rel_grad_err(g_gpu, g_ora, agrad=None):
    """||dg|| / ||g|| (agrad None: the plain north_star metric) or / the Z18 scale."""
    g_gpu = np.asarray(g_gpu, np.float64)
    d = np.linalg.norm(g_gpu - g_ora, axis=-1)
    scale = np.linalg.norm(g_ora, axis=-1) if agrad is None else grad_scale(g_ora, agrad)
    return d / np.maximum(scale, 1e-300)
