"""ctypes binding of the BENCH-ONLY ablation library (include/cstf_ablation.h):
the paper's Fig. 4 ADMM arms (Sec. 5.2).  Argument
marshalling only; libcstf never calls into it."""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(os.path.dirname(_HERE), "lib", "libcstf_ablation.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"libcstf_ablation.so not built ({LIB_PATH}); run `python -m paper_conf_icpp_sohksc24_b200.build`")
_lib = ctypes.CDLL(LIB_PATH)
_lib.cstf_ablation_admm.restype = ctypes.c_int
_lib.cstf_ablation_admm.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                    ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
_lib.cstf_ablation_last_error.restype = ctypes.c_char_p
_lib.cstf_ablation_last_calls.restype = ctypes.c_int64
_lib.cstf_ablation_fp64_peak.restype = ctypes.c_double
_lib.cstf_ablation_fp64_peak.argtypes = [ctypes.c_void_p]

BASELINE, OF, PI, OF_PI = 0, 1, 2, 3
ARMS = {"baseline": BASELINE, "of": OF, "pi": PI, "of_pi": OF_PI}


def admm(arm: int, M, S, H, U, max_iter: int = 10, stream=None) -> dict:
    """One ADMM update (tol = 0, max_iter passes) of the given arm, in place on H, U
    (contiguous float64 CUDA tensors, I x R row-major; S is R x R)."""
    import torch
    I, R = H.shape
    for t in (M, S, H, U):
        assert t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()
    st = np.zeros(6)
    s = stream if stream is not None else torch.cuda.current_stream().cuda_stream
    rc = _lib.cstf_ablation_admm(int(arm), M.data_ptr(), S.data_ptr(), H.data_ptr(), U.data_ptr(), I, R,
                                 int(max_iter), st.ctypes.data, ctypes.c_void_p(s))
    if rc != 0:
        raise RuntimeError("cstf_ablation_admm: " + _lib.cstf_ablation_last_error().decode())
    return dict(iters=int(st[0]), rho=st[1], r_primal=st[2], s_dual=st[3], normH2=st[4], normU2=st[5],
                calls=int(_lib.cstf_ablation_last_calls()))


def fp64_peak(stream=None) -> float:
    """Measured FP64 DMMA peak of the current device (TFLOP/s), cstf_ablation_fp64_peak."""
    import torch
    st = stream if stream is not None else torch.cuda.current_stream()
    v = float(_lib.cstf_ablation_fp64_peak(ctypes.c_void_p(st.cuda_stream)))
    if v <= 0:
        raise RuntimeError("cstf_ablation_fp64_peak failed")
    return v
