"""Small invocations of every kernel family for compute-sanitizer (memcheck, racecheck,
synccheck, initcheck):
    compute-sanitizer --tool memcheck python tools/sanitize_cases.py
Cases: the planted configs[0] factorisation (ADMM tolerance mode: speculative chunks
+ replay), the fixed-iteration protocol (fused Gram epilogue, FNN passes), forced
L2-blocked MTTKRP (one-block batches, persisting window), forced hot-row tables, packed
16-byte records (fast and generic kernels, export), the
R = 64 ADMM with the cp.async row-group prefetch over several groups per warp, HALS /
MU, and the bench-only ablation arms.  Sizes are small: the tools slow kernels 10-100x."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402
from paper_conf_icpp_sohksc24_b200 import binding as B  # noqa: E402


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def main():
    torch.cuda.set_device(0)
    which = sys.argv[1:] or ["planted", "fixed", "l2block", "hot", "packed", "admm64", "hals_mu", "partitioned",
                             "ablation"]
    if "planted" in which:
        p = datagen.planted_tiny(1)
        X = B.cstf_tensor_load_coo(p.dims, p.idx, p.vals)
        F = [cu(f) for f in datagen.perturbed_start(p, 1)]
        B.cstf_factorize(X, F, cu(np.zeros(p.R)), B.make_opts(p.R, outer_iters=3, tol=1e-2, max_iter=10))
        print("planted ok", flush=True)
    if "fixed" in which:
        c = datagen.CONFIGS["enron"].scaled(300, nnz_factor=20000)
        idx, vals = c.generate()
        X = B.cstf_tensor_load_coo(c.dims, idx, vals)
        F = [cu(f) for f in datagen.init_factors(c.dims, 32, 1)]
        B.cstf_factorize(X, F, cu(np.zeros(32)), B.make_opts(32, outer_iters=2, tol=0.0, max_iter=10))
        print("fixed ok", flush=True)
    if "l2block" in which:
        os.environ["CSTF_L2_BLOCK_ROWS"] = "64"
        os.environ["CSTF_L2_BATCH_BYTES"] = "1"
        os.environ["CSTF_L2_PERSIST"] = str(4 << 20)
        dims = (50, 3000, 20)
        idx, vals = datagen.coo(dims, (2, 2, 1), 20000, 41)
        X = B.cstf_tensor_load_coo(dims, idx, vals)
        F = [cu(f) for f in datagen.init_factors(dims, 16, 8)]
        for n in range(3):
            B.cstf_mttkrp(X, n, F, cu(np.zeros((dims[n], 16))))
        for k in ("CSTF_L2_BLOCK_ROWS", "CSTF_L2_BATCH_BYTES", "CSTF_L2_PERSIST"):
            del os.environ[k]
        print("l2block ok", flush=True)
    if "hot" in which:
        os.environ["CSTF_HOT_ROWS"] = "100"
        dims = (60, 2000, 700, 20)
        idx, vals = datagen.coo(dims, (2, 2, 3, 1), 30000, 51)
        X = B.cstf_tensor_load_coo(dims, idx, vals)
        F = [cu(f) for f in datagen.init_factors(dims, 32, 9)]
        for n in range(4):
            B.cstf_mttkrp(X, n, F, cu(np.zeros((dims[n], 32))))
        B.cstf_factorize(X, F, cu(np.zeros(32)), B.make_opts(32, outer_iters=2, tol=0.0, max_iter=4))
        X.export_coo()
        del os.environ["CSTF_HOT_ROWS"]
        print("hot ok", flush=True)
    if "packed" in which:
        # packed 16-byte records forced on every 4-mode copy, hot-row flags in the keys,
        # fast (R = 32) and generic (R = 5) kernels, export
        os.environ["CSTF_PACK"] = "2"
        os.environ["CSTF_HOT_ROWS"] = "100"
        dims = (60, 2000, 700, 20)
        idx, vals = datagen.coo(dims, (2, 2, 3, 1), 30000, 52)
        X = B.cstf_tensor_load_coo(dims, idx, vals)
        assert all(X.record_bytes(n) == 16 for n in range(4))
        for R in (32, 5):
            F = [cu(f) for f in datagen.init_factors(dims, R, 10)]
            for n in range(4):
                B.cstf_mttkrp(X, n, F, cu(np.zeros((dims[n], R))))
        X.export_coo()
        del os.environ["CSTF_PACK"], os.environ["CSTF_HOT_ROWS"]
        print("packed ok", flush=True)
    if "admm64" in which:
        I, R = 20_003, 64          # 2,501 groups over <= 296 CTAs x 4 warps: several groups per warp
        rng = np.random.default_rng(1)
        M, H, U = rng.random((I, R)), rng.random((I, R)), np.zeros((I, R))
        A = rng.random((R, R))
        S = A @ A.T / R
        for tol in (0.0, 1e-2):
            B.cstf_admm_update(cu(M), cu(S), cu(H), cu(U), tol=tol, max_iter=10)
        print("admm64 ok", flush=True)
    if "hals_mu" in which:
        rng = np.random.default_rng(2)
        I, R = 3001, 32
        M, H = rng.random((I, R)), rng.random((I, R))
        A = rng.random((R, R))
        S = A @ A.T / R
        B.cstf_hals_update(cu(M), cu(S), cu(H), sweeps=2)
        B.cstf_mu_update(cu(M), cu(S), cu(H), sweeps=2)
        print("hals_mu ok", flush=True)
    if "partitioned" in which:        # one-part loopback communicator: partitioned store, hot rows, agreement
        os.environ["CSTF_HOT_ROWS"] = "100"
        comm = B.cstf_comm_loopback(1)[0]
        dims = (60, 2000, 700, 20)
        idx, vals = datagen.coo(dims, (2, 2, 3, 1), 30000, 52)
        X = B.cstf_tensor_load_coo(dims, idx, vals, comm=comm)
        F = [cu(f) for f in datagen.init_factors(dims, 32, 9)]
        B.cstf_factorize(X, F, cu(np.zeros(32)), B.make_opts(32, outer_iters=2, tol=0.0, max_iter=4), comm=comm)
        del os.environ["CSTF_HOT_ROWS"]
        print("partitioned ok", flush=True)
    if "ablation" in which:
        from paper_conf_icpp_sohksc24_b200 import ablation as AB
        rng = np.random.default_rng(3)
        I, R = 2001, 32
        A = rng.random((R, R))
        S = cu(A @ A.T / R)
        for arm in range(4):
            AB.admm(arm, cu(rng.random((I, R))), S, cu(rng.random((I, R))), cu(np.zeros((I, R))), max_iter=3)
        print("ablation ok", flush=True)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
