"""Co-run metrics (§6.1; Eyerman & Eeckhout [14], reading A17).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations


def ntt(turnaround, alone):
    """Normalised turnaround time of one kernel: T_shared / T_alone."""
    return turnaround / alone


def antt(turnarounds, alones):
    """Average normalised turnaround time: mean_i T_i^shared / T_i^alone (lower is better)."""
    return sum(t / a for t, a in zip(turnarounds, alones)) / len(alones)


def stp(turnarounds, alones):
    """System throughput: sum_i T_i^alone / T_i^shared (higher is better)."""
    return sum(a / t for t, a in zip(turnarounds, alones))


def natt_gain(antt_base, antt_flep):
    """ANTT improvement of FLEP over a baseline (the paper's 'X' figures)."""
    return antt_base / antt_flep


def hp_speedup(turnaround_base, turnaround_flep):
    """High-priority kernel speedup (Fig. 8)."""
    return turnaround_base / turnaround_flep


def performance_degradation(t_w, t_e):
    """(T_w + T_e) / T_e — the per-kernel quantity HPF's SRPT minimises the sum of."""
    return (t_w + t_e) / t_e


def spatial_overhead(t_flep, t_org):
    """(T_FLEP - T_org) / T_org."""
    return (t_flep - t_org) / t_org


def overhead_reduction(ovh_spatial, ovh_temporal):
    """Reduction of preemption overhead of spatial vs temporal preemption (Fig. 15)."""
    return 1.0 - ovh_spatial / ovh_temporal
