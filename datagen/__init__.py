"""Seeded synthetic inputs for the cSTF hot path (shared by oracle and CUDA path).

This module holds none of the method's arithmetic: it draws indices, values
and initial factors from a counter-based SplitMix64 stream (``gen.c``) and
builds the planted tiny tensor of BASELINE.json ``configs[0]``.  Shapes follow
PAPER.md Table 2 (L917-928); the distributions are DESIGN.md's input recipe
(the paper gives none).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "libdatagen.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gen.c into libdatagen.so (gcc, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-ffp-contract=off",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _get():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, u64, p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p
        lib.datagen_uniform.argtypes = [u64, u64, i64, p]
        lib.datagen_mode_indices.argtypes = [u64, ctypes.c_int, i64, ctypes.c_int, i64, p]
        lib.datagen_values.argtypes = [u64, i64, p]
        lib.datagen_scatter_params.argtypes = [i64, ctypes.POINTER(i64), ctypes.POINTER(i64)]
        _lib = lib
    return _lib


def uniform(seed: int, stream: int, count: int) -> np.ndarray:
    """U[0,1) FP64 draws t = 0..count-1 of (seed, stream)."""
    out = np.empty(count, dtype=np.float64)
    _get().datagen_uniform(seed, stream, count, out.ctypes.data)
    return out


def scatter_params(I: int) -> tuple[int, int]:
    a, b = ctypes.c_int64(), ctypes.c_int64()
    _get().datagen_scatter_params(I, ctypes.byref(a), ctypes.byref(b))
    return a.value, b.value


def coo(dims, gammas, nnz: int, seed: int):
    """Synthetic COO (before coalescing): list of int32 index arrays + FP64 values."""
    lib = _get()
    idx = []
    for n, (I, g) in enumerate(zip(dims, gammas)):
        a = np.empty(nnz, dtype=np.int32)
        lib.datagen_mode_indices(seed, n, int(I), int(g), nnz, a.ctypes.data)
        idx.append(a)
    vals = np.empty(nnz, dtype=np.float64)
    lib.datagen_values(seed, nnz, vals.ctypes.data)
    return idx, vals


def init_factors(dims, R: int, seed: int):
    """Initial factors U[0,1) (stream 1000+n), row-major I_n x R."""
    return [uniform(seed, 1000 + n, int(I) * R).reshape(int(I), R) for n, I in enumerate(dims)]


@dataclass
class Config:
    name: str
    dims: tuple
    gammas: tuple
    nnz: int
    R: int
    seed: int
    note: str = ""
    extra: dict = field(default_factory=dict)

    def scaled(self, factor: float, nnz_factor: float | None = None, name: str | None = None) -> "Config":
        """Same recipe with every mode length divided by `factor` (>= 2 rows) and nnz by nnz_factor."""
        nf = factor if nnz_factor is None else nnz_factor
        dims = tuple(max(2, int(round(I / factor))) for I in self.dims)
        return Config(name or f"{self.name}/{factor:g}", dims, self.gammas,
                      max(1, int(round(self.nnz / nf))), self.R, self.seed, self.note)

    def generate(self):
        return coo(self.dims, self.gammas, self.nnz, self.seed)


# BASELINE.json configs (shapes from PAPER.md Table 2; gamma per mode kind).
CONFIGS = {
    "nell2": Config("nell2", (12_000, 9_000, 29_000), (2, 2, 2), 77_000_000, 32, 2,
                    "NELL-2-shaped 3-mode, 77M nnz, R=32"),
    "enron": Config("enron", (6_000, 5_700, 244_000, 1_200), (2, 2, 3, 1), 54_000_000, 32, 3,
                    "Enron-shaped 4-mode, 54M nnz, R=32"),
    "delicious": Config("delicious", (533_000, 17_300_000, 2_500_000, 1_400), (2, 2, 3, 1),
                        140_000_000, 32, 4, "Delicious-4D-shaped, 140M nnz, R=32"),
    "amazon": Config("amazon", (4_800_000, 1_800_000, 1_800_000), (2, 2, 3), 1_700_000_000, 64, 5,
                     "Amazon-reviews-shaped 3-mode, 1.7B nnz, R=64"),
}


@dataclass
class Planted:
    dims: tuple
    R: int
    idx: list
    vals: np.ndarray
    truth: list


def planted_tiny(seed: int = 1) -> Planted:
    """configs[0]: planted non-negative rank-8 tensor 50x40x30 with exactly 2,000 nnz.

    Mode-1 rows 5r..5r+4 (rows 40..49 empty), mode-2 rows 5r..5r+4, mode-3 support
    10 of 30 per component (seeded); entries U[0.5,1.5) on the supports.  The (i,j)
    blocks of different components are disjoint, so X = sum_r a_r o b_r o c_r has
    8*5*5*10 = 2000 nonzeros, each a single product a_ir*b_jr*c_kr.
    """
    I, J, K, R = 50, 40, 30, 8
    A = np.zeros((I, R)); B = np.zeros((J, R)); C = np.zeros((K, R))
    ua = uniform(seed, 2000, I * R).reshape(I, R)
    ub = uniform(seed, 2001, J * R).reshape(J, R)
    uc = uniform(seed, 2002, K * R).reshape(K, R)
    us = uniform(seed, 2003, R * K)
    supports = []
    for r in range(R):
        A[5 * r:5 * r + 5, r] = 0.5 + ua[5 * r:5 * r + 5, r]
        B[5 * r:5 * r + 5, r] = 0.5 + ub[5 * r:5 * r + 5, r]
        perm = list(range(K))            # seeded partial Fisher-Yates
        for t in range(10):
            s = t + int(us[r * K + t] * (K - t))
            perm[t], perm[s] = perm[s], perm[t]
        sup = sorted(perm[:10])
        supports.append(sup)
        C[sup, r] = 0.5 + uc[sup, r]
    ii, jj, kk, vv = [], [], [], []
    for r in range(R):
        for i in range(5 * r, 5 * r + 5):
            for j in range(5 * r, 5 * r + 5):
                for k in supports[r]:
                    ii.append(i); jj.append(j); kk.append(k)
                    vv.append(A[i, r] * B[j, r] * C[k, r])
    order = np.argsort(uniform(seed, 2004, len(vv)), kind="stable")   # scramble input order
    idx = [np.asarray(x, dtype=np.int32)[order] for x in (ii, jj, kk)]
    vals = np.asarray(vv, dtype=np.float64)[order]
    return Planted((I, J, K), R, idx, vals, [A, B, C])


def perturbed_start(p: Planted, seed: int = 1, eps: float = 0.05):
    """Truth + eps * U[0,1) * max(truth) on every entry (P8 start point)."""
    out = []
    for n, T in enumerate(p.truth):
        u = uniform(seed, 3000 + n, T.size).reshape(T.shape)
        out.append(T + eps * u * T.max())
    return out
