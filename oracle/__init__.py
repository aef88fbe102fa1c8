"""FP64 CPU oracle for the cSTF / AO-ADMM hot path (TEST INFRASTRUCTURE ONLY).

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` leg may import this package.  It shares no code with the
CUDA path (``paper_conf_icpp_sohksc24_b200``) and never consumes its outputs.
The arithmetic lives in ``cstf_oracle.c`` (plain C, FP64, no FMA contraction),
each function citing the PAPER.md passage it follows; this file only marshals
numpy arrays.  See DESIGN.md "Oracle" for the readings D1-D20 and the pins.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cstf_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

OK, EINVAL, ENOMEM, NOT_SPD, NUMERIC = 0, 1, 3, 6, 7
PROX_NONNEG, PROX_IDENTITY, PROX_L1, PROX_NONNEG_L1, PROX_BOX = 0, 1, 2, 3, 4
WARM_SCALED, WARM_NORMALIZED = 0, 1
UPDATE_ADMM, UPDATE_HALS, UPDATE_MU = 0, 1, 2


class OracleError(RuntimeError):
    def __init__(self, code, what):
        super().__init__(f"oracle {what}: status {code}")
        self.code = code


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-ffp-contract=off",
                               "-fno-fast-math", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _get():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        p, i64, i32, d = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
        L.oracle_coalesce.restype = i64
        L.oracle_coalesce.argtypes = [i32, p, i64, p, p, p, p, p, p]
        L.oracle_canonical_hash.restype = ctypes.c_uint64
        L.oracle_canonical_hash.argtypes = [i32, i64, p, p]
        L.oracle_mttkrp.argtypes = [i32, p, i64, p, p, i32, i32, p, p]
        L.oracle_mttkrp_rows.argtypes = [i32, p, i64, p, p, i32, i32, p, i64, p, p]
        L.oracle_gram.argtypes = [i64, i32, p, p]
        L.oracle_hadamard_except.argtypes = [i32, i32, p, i32, p]
        L.oracle_cholesky.argtypes = [i32, p, p]
        L.oracle_admm.argtypes = [i64, i32, p, p, p, p, d, i32, d, i32, d, p, p]
        L.oracle_normalize.argtypes = [i64, i32, p, p]
        L.oracle_hals.argtypes = [i64, i32, p, p, p, i32]
        L.oracle_mu.argtypes = [i64, i32, p, p, p, i32]
        L.oracle_fit.restype = d
        L.oracle_fit.argtypes = [i32, i32, d, i64, p, p, p, p]
        L.oracle_set_threads.argtypes = [i32]
        L.oracle_threads.restype = i32
        L.oracle_factorize.argtypes = [i32, p, i64, p, p, d, i32, i32, d, d, i32, d, i32, i32, i32, d, i32,
                                       p, p, p, p, p, p, p]
        _lib = L
    return _lib


def set_threads(n: int) -> int:
    """OpenMP threads of the oracle's parallel regions (results do not depend on it,
    pin P11); returns the count now in effect."""
    L = _get()
    L.oracle_set_threads(int(n))
    return int(L.oracle_threads())


def threads() -> int:
    return int(_get().oracle_threads())


def _ptrs(arrays, ctype=ctypes.c_void_p):
    return (ctype * len(arrays))(*[a.ctypes.data for a in arrays])


def _c64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _ci32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


class Tensor:
    """Coalesced tensor in canonical order (O1)."""

    def __init__(self, dims, idx, vals, normX2, hash_):
        self.dims = tuple(int(x) for x in dims)
        self.idx = idx
        self.vals = vals
        self.normX2 = normX2
        self.hash = hash_

    @property
    def nmodes(self):
        return len(self.dims)

    @property
    def nnz(self):
        return len(self.vals)


def coalesce(dims, idx, vals) -> Tensor:
    """O1: canonical lexicographic order, duplicates summed, ||X||^2, checksum."""
    L = _get()
    N = len(dims)
    dims_a = np.asarray(dims, dtype=np.int64)
    idx = [_ci32(a) for a in idx]
    vals = _c64(vals)
    nnz = len(vals)
    out_idx = [np.empty(nnz, dtype=np.int32) for _ in range(N)]
    out_vals = np.empty(nnz, dtype=np.float64)
    nx = ctypes.c_double()
    h = ctypes.c_uint64()
    n = L.oracle_coalesce(N, dims_a.ctypes.data, nnz, _ptrs(idx), vals.ctypes.data,
                          _ptrs(out_idx), out_vals.ctypes.data, ctypes.byref(nx), ctypes.byref(h))
    if n < 0:
        raise OracleError(EINVAL, "coalesce")
    return Tensor(dims, [a[:n].copy() for a in out_idx], out_vals[:n].copy(), nx.value, h.value)


def canonical_hash(idx, vals) -> int:
    idx = [_ci32(a) for a in idx]
    vals = _c64(vals)
    return int(_get().oracle_canonical_hash(len(idx), len(vals), _ptrs(idx), vals.ctypes.data))


def mttkrp(X: Tensor, mode: int, factors) -> np.ndarray:
    """O2 (Fig. 2)."""
    R = factors[0].shape[1]
    fs = [_c64(f) for f in factors]
    M = np.empty((X.dims[mode], R))
    dims_a = np.asarray(X.dims, dtype=np.int64)
    st = _get().oracle_mttkrp(X.nmodes, dims_a.ctypes.data, X.nnz, _ptrs(X.idx), X.vals.ctypes.data,
                              mode, R, _ptrs(fs), M.ctypes.data)
    if st:
        raise OracleError(st, "mttkrp")
    return M


def mttkrp_rows(X: Tensor, mode: int, factors, rows) -> np.ndarray:
    R = factors[0].shape[1]
    fs = [_c64(f) for f in factors]
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.empty((len(rows), R))
    dims_a = np.asarray(X.dims, dtype=np.int64)
    st = _get().oracle_mttkrp_rows(X.nmodes, dims_a.ctypes.data, X.nnz, _ptrs(X.idx), X.vals.ctypes.data,
                                   mode, R, _ptrs(fs), len(rows), rows.ctypes.data, out.ctypes.data)
    if st:
        raise OracleError(st, "mttkrp_rows")
    return out


def gram(H) -> np.ndarray:
    """O3: G = H^T H (Alg. 1 l.4/12)."""
    H = _c64(H)
    I, R = H.shape
    G = np.empty((R, R))
    _get().oracle_gram(I, R, H.ctypes.data, G.ctypes.data)
    return G


def hadamard_except(grams, n: int) -> np.ndarray:
    """O4: S = *_{k != n} G^(k) (Alg. 1 l.8)."""
    gs = [_c64(g) for g in grams]
    R = gs[0].shape[0]
    S = np.empty((R, R))
    _get().oracle_hadamard_except(len(gs), R, _ptrs(gs), n, S.ctypes.data)
    return S


def cholesky(A) -> np.ndarray:
    """O6: Cholesky-Banachiewicz, A = L L^T."""
    A = _c64(A)
    R = A.shape[0]
    L = np.empty((R, R))
    st = _get().oracle_cholesky(R, A.ctypes.data, L.ctypes.data)
    if st:
        raise OracleError(st, "cholesky")
    return L


def admm(M, S, H, U, tol=0.0, max_iter=10, rho=0.0, prox=PROX_NONNEG, trace=False, alpha=0.0):
    """O7: Alg. 2 (L550-580). Returns (H, U, stats dict[, trace array])."""
    M = _c64(M); S = _c64(S)
    H = np.array(H, dtype=np.float64, copy=True, order="C")
    U = np.array(U, dtype=np.float64, copy=True, order="C")
    I, R = M.shape
    stats = np.zeros(6)
    tr = np.zeros((max_iter, 4)) if trace else None
    st = _get().oracle_admm(I, R, M.ctypes.data, S.ctypes.data, H.ctypes.data, U.ctypes.data,
                            float(tol), int(max_iter), float(rho), int(prox), float(alpha), stats.ctypes.data,
                            tr.ctypes.data if trace else None)
    if st:
        raise OracleError(st, "admm")
    sd = dict(iters=int(stats[0]), rho=stats[1], r_primal=stats[2], s_dual=stats[3],
              normH2=stats[4], normU2=stats[5])
    if trace:
        return H, U, sd, tr[:sd["iters"]]
    return H, U, sd


def normalize(H):
    """O8: column 2-norms (reading D7); returns (H_normalised, lam)."""
    H = np.array(H, dtype=np.float64, copy=True, order="C")
    I, R = H.shape
    lam = np.empty(R)
    _get().oracle_normalize(I, R, H.ctypes.data, lam.ctypes.data)
    return H, lam


def fit(normX2, M_last, H_last, lam, grams) -> float:
    """O10 (reading D12)."""
    M_last = _c64(M_last); H_last = _c64(H_last); lam = _c64(lam)
    gs = [_c64(g) for g in grams]
    I, R = M_last.shape
    return float(_get().oracle_fit(len(gs), R, float(normX2), I, M_last.ctypes.data,
                                   H_last.ctypes.data, lam.ctypes.data, _ptrs(gs)))


def hals(M, S, H, sweeps=1):
    """f1 HALS (reading D21): column-wise non-negative coordinate updates, in order."""
    M = _c64(M); S = _c64(S)
    H = np.array(H, dtype=np.float64, copy=True, order="C")
    I, R = H.shape
    st = _get().oracle_hals(I, R, M.ctypes.data, S.ctypes.data, H.ctypes.data, int(sweeps))
    if st:
        raise OracleError(st, "hals")
    return H


def mu(M, S, H, sweeps=1):
    """f1 MU (reading D22): h <- h * m / (h S + 1e-16)."""
    M = _c64(M); S = _c64(S)
    H = np.array(H, dtype=np.float64, copy=True, order="C")
    I, R = H.shape
    st = _get().oracle_mu(I, R, M.ctypes.data, S.ctypes.data, H.ctypes.data, int(sweeps))
    if st:
        raise OracleError(st, "mu")
    return H


def factorize(X: Tensor, factors, outer_iters=10, tol=1e-2, max_iter=10, rho=0.0,
              warm=WARM_SCALED, normalize_init=True, prox=PROX_NONNEG, fit_tol=0.0, alpha=0.0,
              update=UPDATE_ADMM):
    """O9/O11: Alg. 1 (L476-506) with readings D4, D6, D11, D13.

    Returns dict(factors, lam (N x R), fit[outer_done], iters[outer_done x N], phase_ms[4],
    trace[outer_done x N x max_iter x 4] of the ADMM sums)."""
    N = X.nmodes
    R = factors[0].shape[1]
    H = [np.array(f, dtype=np.float64, copy=True, order="C") for f in factors]
    lam = np.zeros((N, R))
    fits = np.zeros(outer_iters)
    iters = np.zeros((outer_iters, N), dtype=np.int32)
    done = ctypes.c_int()
    phase = np.zeros(4)
    trace = np.zeros((outer_iters, N, max_iter, 4))
    dims_a = np.asarray(X.dims, dtype=np.int64)
    st = _get().oracle_factorize(N, dims_a.ctypes.data, X.nnz, _ptrs(X.idx), X.vals.ctypes.data,
                                 float(X.normX2), R, int(outer_iters), float(fit_tol), float(tol),
                                 int(max_iter), float(rho), int(warm), int(bool(normalize_init)),
                                 int(prox), float(alpha), int(update), _ptrs(H), lam.ctypes.data, fits.ctypes.data,
                                 iters.ctypes.data, ctypes.byref(done), phase.ctypes.data,
                                 trace.ctypes.data)
    if st:
        raise OracleError(st, "factorize")
    d = done.value
    return dict(factors=H, lam=lam, fit=fits[:d], iters=iters[:d], phase_ms=phase, trace=trace[:d],
                tol=tol)
