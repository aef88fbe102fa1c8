"""Byte / flop accounting for the cSTF hot path (host logic, no GPU).

Two models:
* ``paper_*`` -- the paper's own ADMM cost model, Eq. 3-5:
  W = 19 I R + 2 I R^2 flops, Q = 22 I R + R^2 words per ADMM iteration.
* algorithmic bytes of OUR kernels, the numerator of
  the ``roofline.achieved`` figure bench.py reports:
  - ADMM: every update must read M, H, U and write H, U once: 40 I R bytes
    (FP64).  The streaming form repeats that per inner iteration; the
    row-resident form moves it once per update.
  - MTTKRP: the compulsory traffic of the mode-n nonzero store plus one read of
    every other factor and one write of M.
"""
from __future__ import annotations


def paper_flops_per_iter(I: int, R: int) -> int:
    """Eq. 3 (L667): W = 19IR + 2IR^2."""
    return 19 * I * R + 2 * I * R * R


def paper_words_per_iter(I: int, R: int) -> int:
    """Eq. 4 (L668): Q = 22IR + R^2 (8-byte words)."""
    return 22 * I * R + R * R


def paper_ai(I: int, R: int) -> float:
    """Eq. 5 (L669-671): W / (8 Q), flop per byte."""
    return paper_flops_per_iter(I, R) / (8.0 * paper_words_per_iter(I, R))


def paper_ai_limit(R: int) -> float:
    """Eq. 5 for I >> R (L682): (19 + 2R) / 176."""
    return (19 + 2 * R) / 176.0


def fusion_compute_auxiliary_words(I: int, R: int, fused: bool) -> tuple[int, int]:
    """Sec. 4.3.1 (L823-829): H~ = M + rho (H + U).

    Two DGEAM calls: (H+U) reads 2IR writes IR, then (+M) reads 2IR writes IR.
    Fused: reads M, H, U (3IR), writes IR.  Returns (reads, writes) in words."""
    if fused:
        return 3 * I * R, I * R
    return 4 * I * R, 2 * I * R


def admm_flops_per_row_iter(R: int) -> int:
    """FP64 flops per row per inner iteration (same count as Eq. 3 per row)."""
    return 2 * R * R + 19 * R


def admm_bytes(I: int, R: int) -> int:
    """Compulsory ADMM traffic: read M, H, U; write H, U (FP64)."""
    return 5 * I * R * 8


def mttkrp_bytes(nnz: int, dims, mode: int, R: int) -> int:
    """Compulsory MTTKRP traffic for our mode-sorted store.

    Per nonzero: one FP64 value + one int32 index per other mode; the int64
    row pointer (I_n + 1); one read of each other factor; one write of M."""
    N = len(dims)
    b = nnz * (8 + 4 * (N - 1)) + 8 * (dims[mode] + 1)
    b += sum(dims[k] * R * 8 for k in range(N) if k != mode)
    b += dims[mode] * R * 8
    return b


def mttkrp_flops(nnz: int, N: int, R: int) -> int:
    """(N-2) Hadamard multiplies + 1 scale + 1 add per column per nonzero = N R."""
    return nnz * N * R


def gram_bytes(I: int, R: int) -> int:
    return I * R * 8


def gram_flops(I: int, R: int) -> int:
    """Upper triangle incl. diagonal, 2 flops per multiply-add."""
    return I * R * (R + 1)


def admm_flops_executed(I: int, R: int, k: int, fnn: bool = True, gram: bool = True) -> int:
    """FP64 flops the row-resident kernel (k_admm_dmma) actually executes for one
    update of k passes with tol = 0, as opposed to Eq. 3:
      * the R x R product on DMMA.8x8x4: 2 RP^2 per row and pass (RP = R rounded
        up to a multiple of 8: padded columns are computed);
      * element-wise, FNN passes (every pass but the last with the non-negativity
        prox): x = H~ + w (DADD) and rho |x| + M (DFMA) = 3 flops per element
        (the prox, |x| and the dual are sign-bit integer operations);
      * the last pass (plain epilogue with the residual sums): A operand
        (DADD + DFMA), x, H' - x, two residual differences, four DFMA sums
        = 13 flops per element;
      * the fused Gram epilogue: NT(NT+1)/2 tile pairs x 2 DMMA.8x8x4 per 8 rows.
    Without FNN every pass costs the plain epilogue's A operand + x + dual = 5
    flops per element, the last pass 13."""
    RP = (R + 7) // 8 * 8
    NT = RP // 8
    prod = 2 * RP * RP * k
    if fnn and k > 1:
        elem = 3 * R * (k - 1) + 13 * R
    else:
        elem = 5 * R * max(k - 1, 0) + 13 * R
    g = (NT * (NT + 1) // 2) * 2 * (8 * 8 * 4 * 2) / 8 if gram else 0
    return int(I * (prod + elem + g))
