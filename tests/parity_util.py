"""Shared comparison helpers for GPU-vs-oracle parity (test logic, no method arithmetic)."""
import numpy as np

TIE_MARGIN = 1e-12


def stop_margin(trace_row, eps):
    """Reading U2: mu = min(eps nH - r, eps nU - s) / (eps (nH + nU)) at one ADMM pass."""
    r, s, nH, nU = trace_row
    den = eps * (nH + nU)
    if den == 0.0:
        return 0.0
    return min(eps * nH - r, eps * nU - s) / den


def compare_iteration_counts(gpu_iters, orc, eps):
    """ADMM iteration counts must be equal per (outer iteration, mode).  A mismatch
    is accepted only as a tie (U2): at the decisive pass min(k_gpu, k_orc) the
    oracle's margin |mu| < TIE_MARGIN.  After the first tie the trajectories are
    different rounding paths and counts are no longer compared.
    Returns (n_compared, first_tie or None)."""
    oi = orc["iters"]
    tr = orc["trace"]
    assert gpu_iters.shape == oi.shape, (gpu_iters.shape, oi.shape)
    n = 0
    for t in range(oi.shape[0]):
        for m in range(oi.shape[1]):
            kg, ko = int(gpu_iters[t, m]), int(oi[t, m])
            if kg != ko:
                j = min(kg, ko) - 1
                mu = stop_margin(tr[t, m, j], eps)
                assert abs(mu) < TIE_MARGIN, (
                    f"ADMM iteration count differs at outer {t} mode {m}: gpu {kg} oracle {ko}, "
                    f"margin {mu:.3e} is not a tie")
                return n, (t, m, mu)
            n += 1
    return n, None


def compare_all_iteration_counts(gpu_iters, orc, eps):
    """Every (outer iteration, mode) pair: the counts are equal, or the mismatch is a
    tie (U2: |mu| < TIE_MARGIN at the oracle's pass min(k_gpu, k_orc)).  Unlike
    compare_iteration_counts this keeps comparing after a tie (both trajectories
    stay within rounding of each other once they sit at the fixed point).
    Returns (n_equal, n_ties)."""
    oi = orc["iters"]
    tr = orc["trace"]
    assert gpu_iters.shape == oi.shape, (gpu_iters.shape, oi.shape)
    eq = ties = 0
    for t in range(oi.shape[0]):
        for m in range(oi.shape[1]):
            kg, ko = int(gpu_iters[t, m]), int(oi[t, m])
            if kg == ko:
                eq += 1
                continue
            mu = stop_margin(tr[t, m, min(kg, ko) - 1], eps)
            assert abs(mu) < TIE_MARGIN, (
                f"ADMM iteration count differs at outer {t} mode {m}: gpu {kg} oracle {ko}, "
                f"margin {mu:.3e} is not a tie")
            ties += 1
    return eq, ties
