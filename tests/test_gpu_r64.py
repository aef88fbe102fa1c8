"""GPU parity on the paths the Amazon-shaped configuration (BASELINE configs[4],
R = 64; PAPER.md L907-908 ranks {16, 32, 64}, Table 2) takes, at sizes the
oracle finishes in seconds:
  * the R = 64 ADMM kernel with several 8-row groups per warp, so the cp.async
    next-group prefetch (PREF) actually loads (tol = 0 and tol > 0 with replay);
  * a scaled Amazon-shaped factorisation at R = 64 with L2-blocked mode copies,
    one-block batches and persisting-L2 windows forced small, against the oracle;
  * factorize with fit_tol > 0 (D11) and with normalize_init = 0 (D6) against
    the oracle.
Tolerances as in test_gpu_parity.py (north_star): fixed-iteration ADMM <= 1e-9
normwise; factorize fit <= 1e-6 relative, factors <= 1e-6, ADMM counts equal.
"""
import numpy as np
import pytest

import datagen
import oracle
from parity_util import compare_iteration_counts

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-9


@pytest.fixture(scope="module")
def B():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_sohksc24_b200 import binding
    return binding


def normwise(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    den = np.max(np.abs(b)) if b.size else 0.0
    return float(np.max(np.abs(a - b)) / (den if den > 0 else 1.0)) if b.size else 0.0


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def admm_inputs(I, R, seed, nmodes=3):
    Fs = [oracle.normalize(datagen.uniform(seed, 10 + k, 200 * R).reshape(200, R))[0] for k in range(nmodes)]
    S = oracle.hadamard_except([oracle.gram(F) for F in Fs], 0)
    M = datagen.uniform(seed, 20, I * R).reshape(I, R) * 2.0 - 0.5
    H = datagen.uniform(seed, 21, I * R).reshape(I, R)
    U = (datagen.uniform(seed, 22, I * R).reshape(I, R) - 0.5) * 0.1
    return M, S, H, U


@pytest.mark.parametrize("pref", ["1", "0"])
@pytest.mark.parametrize("max_iter,tol", [(10, 0.0), (3, 0.0), (30, 1e-2), (40, 1e-3)])
def test_admm_r64_several_groups_per_warp(B, pref, max_iter, tol, monkeypatch):
    """I = 60,001 rows at R = 64: 7,501 row groups over at most 148 x 2 CTAs x 4 warps,
    so every warp runs >= 6 groups and the PREF kernel's next-group prefetch fires
    (the last group is ragged).  tol > 0 runs speculative chunks + exact replay."""
    monkeypatch.setenv("CSTF_ADMM_PREF", pref)
    I, R = 60_001, 64
    M, S, H, U = admm_inputs(I, R, 64 + max_iter)
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=tol, max_iter=max_iter)
    Hr, Ur, sr, tr = oracle.admm(M, S, H, U, tol=tol, max_iter=max_iter, trace=True)
    assert st["iters"] == sr["iters"], (st["iters"], sr["iters"])
    if tol == 0.0:
        assert sr["iters"] == max_iter
    else:
        assert sr["iters"] < max_iter            # the replay path (stop inside a chunk) is taken
    assert normwise(host(Hd), Hr) <= TOL
    assert normwise(host(Ud), Ur) <= TOL
    for k in ("rho", "r_primal", "s_dual", "normH2", "normU2"):
        assert st[k] == pytest.approx(sr[k], rel=1e-9, abs=1e-300), k


def test_admm_r64_prefetch_bit_identical(B, monkeypatch):
    """The prefetching and the plain R = 64 kernels run the same arithmetic."""
    I, R = 50_003, 64
    M, S, H, U = admm_inputs(I, R, 5)
    outs = []
    for pref in ("1", "0"):
        monkeypatch.setenv("CSTF_ADMM_PREF", pref)
        Hd, Ud = cu(H), cu(U)
        B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=10)
        outs.append((host(Hd).tobytes(), host(Ud).tobytes()))
    assert outs[0] == outs[1]


def amazon_small():
    """Amazon-shaped (4.8M x 1.8M x 1.8M, gammas 2/2/3) divided by 200 per mode,
    ~2M nonzeros: 24,000 x 9,000 x 9,000."""
    return datagen.CONFIGS["amazon"].scaled(200, nnz_factor=850)


@pytest.fixture(scope="module")
def amazon_case():
    c = amazon_small()
    idx, vals = c.generate()
    return c, idx, vals, oracle.coalesce(c.dims, idx, vals)


@pytest.mark.parametrize("tol,outer", [(1e-2, 3), (0.0, 2)])
def test_factorize_amazon_shaped_r64_l2_blocked(B, amazon_case, tol, outer, monkeypatch):
    """configs[4] in small at R = 64: every mode copy L2-blocked (1,000-row blocks of the
    longest other factor, forced), one-block batches with a persisting L2 window on each
    slab (forced), the R = 64 PREF ADMM with several groups per warp, and the
    non-fused R = 64 Gram; against the oracle."""
    c, idx, vals, ref = amazon_case
    R = 64
    monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "1000")
    monkeypatch.setenv("CSTF_L2_PERSIST", str(8 << 20))
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    assert X.info()["hash"] == ref.hash
    for n in range(3):
        nblk, rows, bm = X.layout(n)
        assert nblk > 1 and rows == 1000, (n, nblk, rows, bm)
    if tol == 0.0:
        monkeypatch.setenv("CSTF_L2_BATCH_BYTES", "1")          # one block per batch
    start = datagen.init_factors(c.dims, R, c.seed)
    orc = oracle.factorize(ref, start, outer_iters=outer, tol=tol, max_iter=10)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=outer, tol=tol, max_iter=10))
    n, tie = compare_iteration_counts(gpu["iters"], orc, tol if tol > 0 else 1e-2)
    assert tie is None, tie
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(host(a), b) <= 1e-6
    assert normwise(host(lam), orc["lam"][-1]) <= 1e-6


def test_mttkrp_amazon_shaped_r64_every_mode(B, amazon_case, monkeypatch):
    """MTTKRP of every mode at R = 64 on the blocked Amazon-shaped copies (forced) and on
    the default layout, against the oracle; repeatable bit for bit."""
    c, idx, vals, ref = amazon_case
    R = 64
    F = datagen.init_factors(c.dims, R, 11)
    Fd = [cu(f) for f in F]
    for rows in ("1000", None):
        if rows:
            monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", rows)
        else:
            monkeypatch.delenv("CSTF_L2_BLOCK_ROWS", raising=False)
        X = B.cstf_tensor_load_coo(c.dims, idx, vals)
        for n in range(3):
            M = cu(np.full((c.dims[n], R), np.nan))
            B.cstf_mttkrp(X, n, Fd, M)
            first = host(M).copy()
            B.cstf_mttkrp(X, n, Fd, M)
            assert np.array_equal(host(M), first), (rows, n)
            assert normwise(first, oracle.mttkrp(ref, n, F)) <= TOL, (rows, n)


@pytest.mark.parametrize("R", [8, 32])
def test_factorize_fit_tol_vs_oracle(B, R):
    """D11 on the device path against the oracle: fit_tol chosen from the oracle's
    fixed-count fits so the stop is well separated; same stop index, same fits."""
    c = datagen.CONFIGS["enron"].scaled(60, nnz_factor=2000)
    idx, vals = c.generate()
    ref = oracle.coalesce(c.dims, idx, vals)
    start = datagen.init_factors(c.dims, R, 3)
    T = 8
    full = oracle.factorize(ref, start, outer_iters=T, tol=0.0, max_iter=10)
    d = np.abs(np.diff(full["fit"]))
    tstar = next(t for t in range(2, T) if d[t - 1] < np.min(d[:t - 1]))
    lo, hi = d[tstar - 1], np.min(d[:tstar - 1])
    assert hi / lo > 1.5, "stop not well separated"
    fit_tol = np.sqrt(lo * hi)
    orc = oracle.factorize(ref, start, outer_iters=T, tol=0.0, max_iter=10, fit_tol=fit_tol)
    assert len(orc["fit"]) == tstar + 1
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=T, tol=0.0, max_iter=10, fit_tol=fit_tol))
    assert gpu["outer_done"] == tstar + 1
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(host(a), b) <= 1e-6


@pytest.mark.parametrize("warm", [0, 1])
def test_factorize_unnormalised_start_vs_oracle(B, warm):
    """normalize_init = 0 (D6 off: raw factors, lambda = 1) on the device path against the
    oracle, both warm-start readings; raw factors scaled far from unit norm."""
    c = datagen.CONFIGS["nell2"].scaled(40, nnz_factor=800)
    idx, vals = c.generate()
    ref = oracle.coalesce(c.dims, idx, vals)
    R = 16
    start = [f * (0.2 + 5.0 * datagen.uniform(7, 90 + k, R)) for k, f in enumerate(datagen.init_factors(c.dims, R, 4))]
    orc = oracle.factorize(ref, start, outer_iters=4, tol=1e-2, max_iter=10, normalize_init=False, warm=warm)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=4, tol=1e-2, max_iter=10, normalize_init=False,
                                                  warm=warm))
    n, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert tie is None, tie
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(host(a), b) <= 1e-6
