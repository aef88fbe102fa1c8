"""B200-native constrained sparse tensor factorisation (cSTF) with AO-ADMM.

Soh, Kannan, Sao, Choi, "Accelerating Constrained Sparse Tensor Factorization
on Massively Parallel Architectures", ICPP '24.  The hot path (sparse MTTKRP,
Gram/Cholesky/inverse, fused ADMM update, normalisation, fit) runs in
hand-written sm_100a CUDA kernels behind the C ABI declared in
``include/cstf.h`` (``libcstf.so``).  ``binding`` is a thin ctypes layer with
the same names; PyTorch only provides device memory, streams and process
groups.  There is no CPU fallback: if ``libcstf.so`` is missing, importing
``binding`` raises.
"""
from . import costmodel  # noqa: F401  (pure host logic)

__all__ = ["costmodel"]
