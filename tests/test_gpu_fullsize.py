"""Full-size parity at configs[1] (NELL-2-shaped,
77M nonzeros, R = 32, eps = 0, 10 inner passes) on sampled outputs the oracle
can compute one by one, plus one complete outer iteration end to end; the same
at configs[3] (Delicious-shaped, 140M nonzeros: the bench default) below."""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-9


def normwise(a, b):
    den = np.max(np.abs(b))
    return float(np.max(np.abs(np.asarray(a) - np.asarray(b))) / (den if den > 0 else 1.0))


@pytest.fixture(scope="module")
def full():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_sohksc24_b200 import binding as B
    c = datagen.CONFIGS["nell2"]
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    ref = oracle.coalesce(c.dims, idx, vals)
    F = datagen.init_factors(c.dims, c.R, c.seed)
    return B, c, X, ref, F


def test_fullsize_store(full):
    B, c, X, ref, F = full
    info = X.info()
    assert info["nnz"] == ref.nnz and info["hash"] == ref.hash
    assert info["normX2"] == pytest.approx(ref.normX2, rel=1e-12)


def test_fullsize_mttkrp_sampled_rows(full):
    B, c, X, ref, F = full
    rng = np.random.default_rng(0)
    Fd = [torch.from_numpy(f).cuda() for f in F]
    for n, I in enumerate(c.dims):
        counts = np.bincount(ref.idx[n], minlength=I)
        rows = np.unique(np.concatenate([rng.integers(0, I, 200), [np.argmax(counts), np.argmin(counts), 0, I - 1]]))
        M = torch.full((I, c.R), float("nan"), dtype=torch.float64, device="cuda")
        B.cstf_mttkrp(X, n, Fd, M)
        torch.cuda.synchronize()
        got = M.cpu().numpy()[rows]
        want = oracle.mttkrp_rows(ref, n, F, rows)
        assert normwise(got, want) <= TOL, n
        assert not np.isnan(M.cpu().numpy()).any()


def test_fullsize_admm_sampled_rows(full):
    """The row-resident ADMM at the largest NELL-2 mode (29K rows, R = 32, 10 passes)."""
    B, c, X, ref, F = full
    I, R = c.dims[2], c.R
    Fs = [oracle.normalize(f)[0] for f in F]
    S = oracle.hadamard_except([oracle.gram(f) for f in Fs], 2)
    M = datagen.uniform(9, 1, I * R).reshape(I, R) * 100.0 - 20.0
    H = datagen.uniform(9, 2, I * R).reshape(I, R)
    U = np.zeros((I, R))
    Hd, Ud = torch.from_numpy(H.copy()).cuda(), torch.from_numpy(U.copy()).cuda()
    B.cstf_admm_update(torch.from_numpy(M).cuda(), torch.from_numpy(S).cuda(), Hd, Ud, tol=0.0, max_iter=10)
    rows = np.random.default_rng(1).choice(I, 300, replace=False)
    Hr, Ur, _ = oracle.admm(M[rows], S, H[rows], U[rows], tol=0.0, max_iter=10)   # rows are independent
    torch.cuda.synchronize()
    assert normwise(Hd.cpu().numpy()[rows], Hr) <= TOL
    assert normwise(Ud.cpu().numpy()[rows], Ur) <= TOL


def test_fullsize_one_outer_iteration(full):
    """One outer iteration of the bench protocol end to end: fit and factors vs the oracle."""
    B, c, X, ref, F = full
    Fd = [torch.from_numpy(f.copy()).cuda() for f in F]
    lam = torch.zeros(c.R, dtype=torch.float64, device="cuda")
    rep = B.cstf_factorize(X, Fd, lam, B.make_opts(c.R, outer_iters=1, tol=0.0, max_iter=10))
    orc = oracle.factorize(ref, F, outer_iters=1, tol=0.0, max_iter=10)
    assert abs(rep["fit"][0] - orc["fit"][0]) <= 1e-6 * abs(orc["fit"][0])
    for a, b in zip(Fd, orc["factors"]):
        assert normwise(a.cpu().numpy(), b) <= 1e-6
    assert normwise(lam.cpu().numpy(), orc["lam"][-1]) <= 1e-6


@pytest.fixture(scope="module")
def delicious():
    """configs[3] (Delicious-shaped, 140M nonzeros, R = 32): the copy of mode 4
    is L2-blocked by default (short output mode, 4.4 GB factor of mode 2)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_sohksc24_b200 import binding as B
    c = datagen.CONFIGS["delicious"]
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    ref = oracle.coalesce(c.dims, idx, vals)
    del idx, vals
    F = datagen.init_factors(c.dims, c.R, c.seed)
    yield B, c, X, ref, F
    X.free()


def test_fullsize_delicious_mttkrp_sampled_rows(delicious):
    B, c, X, ref, F = delicious
    info = X.info()
    assert info["nnz"] == ref.nnz and info["hash"] == ref.hash
    assert [X.layout(n)[0] > 1 for n in range(4)] == [False, False, False, True]
    rng = np.random.default_rng(1)
    Fd = [torch.from_numpy(f).cuda() for f in F]
    for n, I in enumerate(c.dims):
        counts = np.bincount(ref.idx[n], minlength=I)
        k = 12 if n == 3 else 100        # mode-4 rows hold ~100K nonzeros each
        rows = np.unique(np.concatenate([rng.integers(0, I, k), [np.argmax(counts), np.argmin(counts), 0, I - 1]]))
        M = torch.full((I, c.R), float("nan"), dtype=torch.float64, device="cuda")
        B.cstf_mttkrp(X, n, Fd, M)
        torch.cuda.synchronize()
        got = M[torch.from_numpy(rows).cuda()].cpu().numpy()
        want = oracle.mttkrp_rows(ref, n, F, rows)
        assert normwise(got, want) <= TOL, n
        assert not torch.isnan(M).any().item()
        del M


def test_fullsize_delicious_one_outer_iteration(delicious):
    """configs[3] at full size in the bench's launch configuration (default layout:
    hot-row tables, L2-blocked mode 4; eps = 0, 10 passes): one outer iteration end to
    end against the oracle (~40 s of CPU work) -- fit, factors and lambda <= 1e-6."""
    B, c, X, ref, F = delicious
    Fd = [torch.from_numpy(f.copy()).cuda() for f in F]
    lam = torch.zeros(c.R, dtype=torch.float64, device="cuda")
    rep = B.cstf_factorize(X, Fd, lam, B.make_opts(c.R, outer_iters=1, tol=0.0, max_iter=10))
    orc = oracle.factorize(ref, F, outer_iters=1, tol=0.0, max_iter=10)
    assert abs(rep["fit"][0] - orc["fit"][0]) <= 1e-6 * abs(orc["fit"][0])
    for a, b in zip(Fd, orc["factors"]):
        assert normwise(a.cpu().numpy(), b) <= 1e-6
    assert normwise(lam.cpu().numpy(), orc["lam"][-1]) <= 1e-6
