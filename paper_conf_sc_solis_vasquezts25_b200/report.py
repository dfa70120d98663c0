"""Measurement helpers: the paper's Amdahl model and the algorithmic work model.

amdahl_speedup: Eq 6, predicted T_baseline / T_TCEC = 1 / (f/S + (1 - f)),
with f = f_eff and S = TC / SIMT peak ratio.
"""
from __future__ import annotations


def amdahl_speedup(f: float, S: float) -> float:
    return 1.0 / (f / S + (1.0 - f))
