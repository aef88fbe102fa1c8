"""GPU parity: the CUDA path (through the C ABI) against the FP64 oracle on the
same seeded inputs.  Tolerances (north_star):
  integer / index / order work ........ bit-exact (canonical order, checksum)
  MTTKRP, fixed-iteration ADMM ........ normwise max rel <= 1e-9 (reading D18)
  Gram / normalize ..................... <= 1e-12
  end-to-end fit (10 outer iterations) . rel diff <= 1e-6, ADMM iteration counts equal
"""
import numpy as np
import pytest

import datagen
import oracle
from parity_util import compare_all_iteration_counts, compare_iteration_counts

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


def random_coo(seed, dims, nnz, dup_frac=0.2):
    rng = np.random.default_rng(seed)
    idx = [rng.integers(0, I, nnz).astype(np.int32) for I in dims]
    nd = int(nnz * dup_frac)
    if nd:
        s, d = rng.integers(0, nnz, nd), rng.integers(0, nnz, nd)
        for a in idx:
            a[d] = a[s]
    vals = rng.random(nnz) + 0.1
    vals[rng.random(nnz) < 0.05] *= -1
    vals[rng.random(nnz) < 0.02] = 0.0
    return idx, vals


STORE_CASES = [
    ("3mode-dups", (40, 31, 17), 5000, 1),
    ("4mode-dups", (9, 8, 7, 6), 3000, 2),
    ("2mode", (100, 77), 2000, 3),
    ("unit-dim", (1, 50, 1), 300, 4),
    ("wide-keys", (2_000_000_000, 1_500_000_000, 1_000_000_000), 20000, 5),   # > 64 key bits
]


@pytest.mark.parametrize("name,dims,nnz,seed", STORE_CASES)
def test_store_canonical_order_bit_exact(B, name, dims, nnz, seed):
    idx, vals = random_coo(seed, dims, nnz, dup_frac=0.0 if name == "wide-keys" else 0.3)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    info = X.info()
    assert info["nnz"] == ref.nnz
    assert info["hash"] == ref.hash
    gi, gv = X.export_coo()
    for a, b in zip(gi, ref.idx):
        assert np.array_equal(a, b)
    assert np.array_equal(gv, ref.vals)                    # duplicates summed in input order
    assert info["normX2"] == pytest.approx(ref.normX2, rel=1e-13)


def test_store_empty_and_single(B):
    X = B.cstf_tensor_load_coo((4, 5, 6), [np.zeros(0, np.int32)] * 3, np.zeros(0))
    assert X.info()["nnz"] == 0
    F = [cu(np.ones((I, 3))) for I in (4, 5, 6)]
    M = cu(np.full((4, 3), 7.0))
    B.cstf_mttkrp(X, 0, F, M)
    assert np.all(host(M) == 0.0)
    X1 = B.cstf_tensor_load_coo((4, 5, 6), [np.array([3], np.int32), np.array([1], np.int32), np.array([5], np.int32)],
                                np.array([2.5]))
    M = cu(np.zeros((4, 3)))
    B.cstf_mttkrp(X1, 0, F, M)
    assert np.array_equal(host(M), np.array([[0, 0, 0]] * 3 + [[2.5] * 3], dtype=float))


def test_store_rejects_out_of_range(B):
    with pytest.raises(B.CstfError) as e:
        B.cstf_tensor_load_coo((3, 3), [np.array([0, 3], np.int32), np.array([0, 1], np.int32)], np.ones(2))
    assert e.value.status == B.CSTF_ERR_INVALID_ARG


MTTKRP_CASES = [
    ((300, 200, 500), (2, 2, 3), 40000, 7),
    ((60, 5000, 40, 30), (2, 3, 1, 2), 60000, 8),
    ((1000, 900), (3, 1), 30000, 9),
    ((50, 40, 30, 20, 10), (1, 2, 1, 2, 1), 8000, 10),
]


@pytest.mark.parametrize("case", MTTKRP_CASES)
@pytest.mark.parametrize("R", [1, 5, 16, 32, 33, 64, 100, 128])
def test_mttkrp_parity(B, case, R):
    dims, gam, nnz, seed = case
    idx, vals = datagen.coo(dims, gam, nnz, seed)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    F = datagen.init_factors(dims, R, seed)
    Fd = [cu(f) for f in F]
    for n in range(len(dims)):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        want = oracle.mttkrp(ref, n, F)
        assert normwise(host(M), want) <= TOL, (n, R)


@pytest.mark.parametrize("gl", ["0", "8"])
@pytest.mark.parametrize("case", [("3mode", (300, 211, 97), 60000), ("4mode", (40, 37, 53, 29), 50000)])
def test_mttkrp_group_width_variants(B, gl, case, monkeypatch):
    """Both lane-group widths of the R = 32 fast path (16 lanes x 16 B and 8 lanes x 32 B,
    chosen by factor size in production) against the oracle, forced per call."""
    monkeypatch.setenv("CSTF_MTTKRP_G", gl)
    name, dims, nnz = case
    idx, vals = random_coo(len(dims) * 7 + int(gl), dims, nnz, dup_frac=0.05)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    Xo = oracle.coalesce(dims, idx, vals)
    F = [datagen.uniform(3, 40 + k, I * 32).reshape(I, 32) for k, I in enumerate(dims)]
    Fd = [cu(f) for f in F]
    for n in range(len(dims)):
        M = cu(np.full((dims[n], 32), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        assert normwise(host(M), oracle.mttkrp(Xo, n, F)) <= TOL, (n, gl)


def test_mttkrp_heavy_row_spans_many_chunks(B):
    """One row holding most nonzeros (carry fix-up across many chunks) + empty rows."""
    rng = np.random.default_rng(3)
    nnz = 300_000
    i = np.where(rng.random(nnz) < 0.9, 7, rng.integers(0, 50, nnz)).astype(np.int32)
    i[i == 3] = 4                                            # row 3 empty
    j = rng.integers(0, 400, nnz).astype(np.int32)
    k = rng.integers(0, 300, nnz).astype(np.int32)
    dims = (50, 400, 300)
    vals = rng.random(nnz)
    X = B.cstf_tensor_load_coo(dims, [i, j, k], vals)
    ref = oracle.coalesce(dims, [i, j, k], vals)
    F = [rng.random((I, 32)) for I in dims]
    M = cu(np.full((50, 32), np.nan))
    B.cstf_mttkrp(X, 0, [cu(f) for f in F], M)
    got = host(M)
    assert np.all(got[3] == 0.0)
    assert normwise(got, oracle.mttkrp(ref, 0, F)) <= TOL


def test_mttkrp_deterministic(B):
    dims = (300, 200, 500)
    idx, vals = datagen.coo(dims, (2, 2, 3), 40000, 7)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    F = [cu(f) for f in datagen.init_factors(dims, 32, 7)]
    outs = []
    for _ in range(3):
        M = cu(np.zeros((500, 32)))
        B.cstf_mttkrp(X, 2, F, M)
        outs.append(host(M))
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[1], outs[2])


@pytest.mark.parametrize("dmma", ["1", "0"])
@pytest.mark.parametrize("I,R", [(0, 8), (1, 1), (7, 5), (1000, 13), (100003, 32), (4097, 40), (250001, 64),
                                 (999, 65)])
def test_gram_paths(B, I, R, dmma, monkeypatch):
    """cstf_gram on the DMMA path (R <= 64) and on the DFMA register-tile kernel, ragged
    row counts and ranks, against the oracle's Gram; repeatable bit for bit."""
    monkeypatch.setenv("CSTF_GRAM_DMMA", dmma)
    H = datagen.uniform(9, 78, I * R).reshape(I, R) - 0.25
    Hd = cu(H)
    G = cu(np.full((R, R), np.nan))
    B.cstf_gram(Hd, G)
    first = host(G).copy()
    B.cstf_gram(Hd, G)
    assert np.array_equal(host(G), first)
    want = oracle.gram(H) if I > 0 else np.zeros((R, R))
    assert normwise(first, want) <= 1e-12 if I > 0 else np.array_equal(first, want)
    assert np.array_equal(first, first.T)


@pytest.mark.parametrize("I,R", [(1, 4), (1000, 8), (4099, 32), (777, 64), (300, 100), (5000, 3)])
def test_gram_and_normalize(B, I, R):
    H = datagen.uniform(5, 77, I * R).reshape(I, R)
    H[:, R // 2] = 0.0
    G = cu(np.zeros((R, R)))
    B.cstf_gram(cu(H), G)
    assert normwise(host(G), oracle.gram(H)) <= 1e-12
    Hd = cu(H)
    lam = cu(np.zeros(R))
    G2 = cu(np.zeros((R, R)))
    B.cstf_normalize(Hd, lam, G2)
    Hn, lam_ref = oracle.normalize(H)
    assert normwise(host(lam), lam_ref) <= 1e-12
    assert normwise(host(Hd), Hn) <= 1e-12
    assert host(lam)[R // 2] == 0.0 and np.all(host(Hd)[:, R // 2] == 0.0)
    assert normwise(host(G2), oracle.gram(Hn)) <= 1e-12


@pytest.mark.parametrize("R", [32, 7])
def test_normalize_division_exact(B, R):
    """The column scaling divides by lambda through the rounded reciprocal plus one fma
    correction (dense.cu div_by): bit for bit IEEE x / lambda, checked against numpy's
    division with the returned lambda on values spread over 2^-60 .. 2^60 (plus zeros,
    negatives and a zero column), for the paired (even R) and scalar kernels."""
    I = 200_003
    H = datagen.uniform(6, 78, I * R).reshape(I, R) - 0.3
    H *= np.exp2(np.floor(datagen.uniform(6, 79, I * R) * 120.0 - 60.0)).reshape(I, R)
    H[::97, 1] = 0.0
    H[:, R - 1] = 0.0
    Hd = cu(H)
    lam = cu(np.zeros(R))
    B.cstf_normalize(Hd, lam, cu(np.zeros((R, R))))
    l = host(lam)
    want = H.copy()
    nz = l > 0
    want[:, nz] = H[:, nz] / l[nz]
    assert np.array_equal(host(Hd), want)


def admm_inputs(I, R, seed, nmodes=3):
    """M, S, H, U shaped like a real update: S = Hadamard of Grams of normalised factors."""
    Fs = [oracle.normalize(datagen.uniform(seed, 10 + k, 200 * R).reshape(200, R))[0] for k in range(nmodes)]
    S = oracle.hadamard_except([oracle.gram(F) for F in Fs], 0)
    M = datagen.uniform(seed, 20, I * R).reshape(I, R) * 2.0 - 0.5
    H = datagen.uniform(seed, 21, I * R).reshape(I, R)
    U = (datagen.uniform(seed, 22, I * R).reshape(I, R) - 0.5) * 0.1
    return M, S, H, U


@pytest.mark.parametrize("variant", [0, 1, 2])
@pytest.mark.parametrize("I,R", [(1, 8), (1003, 3), (4097, 8), (2049, 16), (3001, 32), (1500, 40), (999, 64),
                                 (600, 65), (300, 128)])
def test_admm_fixed_iterations(B, variant, I, R):
    M, S, H, U = admm_inputs(I, R, R + I)
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=10, variant=variant)
    Hr, Ur, sr = oracle.admm(M, S, H, U, tol=0.0, max_iter=10)
    assert st["iters"] == sr["iters"] == 10
    assert normwise(host(Hd), Hr) <= TOL
    assert normwise(host(Ud), Ur) <= TOL
    for k in ("rho", "r_primal", "s_dual", "normH2", "normU2"):
        assert st[k] == pytest.approx(sr[k], rel=1e-9, abs=1e-300), k


@pytest.mark.parametrize("ireg,pref", [("0", "0"), ("1", "0"), ("1", "1")])
@pytest.mark.parametrize("max_iter", [3, 10])
def test_admm_inv_placement_variants(B, ireg, pref, max_iter, monkeypatch):
    """R = 32 ADMM with the Inv fragments in SMEM and in registers, with and without the
    cp.async row-group prefetch (forced per call); ragged row count (2501)."""
    monkeypatch.setenv("CSTF_ADMM_IREG", ireg)
    monkeypatch.setenv("CSTF_ADMM_PREF", pref)
    M, S, H, U = admm_inputs(2501, 32, 17)
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=max_iter)
    Hr, Ur, sr = oracle.admm(M, S, H, U, tol=0.0, max_iter=max_iter)
    assert st["iters"] == sr["iters"] == max_iter
    assert normwise(host(Hd), Hr) <= TOL and normwise(host(Ud), Ur) <= TOL


@pytest.mark.parametrize("R,ireg", [(8, "0"), (24, "0"), (32, "0"), (32, "1"), (40, "0"), (64, "0")])
@pytest.mark.parametrize("max_iter,tol", [(2, 0.0), (10, 0.0), (17, 0.0), (30, 1e-2)])
def test_admm_fnn_passes_bit_identical(B, R, ireg, max_iter, tol, monkeypatch):
    """The sign-bit (FNN) passes reproduce the plain epilogue bit for bit, including
    signed zeros in the incoming H and U and replayed chunks (tol > 0)."""
    monkeypatch.setenv("CSTF_ADMM_IREG", ireg)
    M, S, H, U = admm_inputs(1203, R, 3 * R + max_iter)
    H[::7] = 0.0
    U[::5] = 0.0
    U[1::9] = -0.0
    H[2::11] = -0.0
    outs = []
    for fnn in ("1", "0"):
        monkeypatch.setenv("CSTF_ADMM_FNN", fnn)
        Hd, Ud = cu(H), cu(U)
        st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=tol, max_iter=max_iter)
        outs.append((host(Hd).tobytes(), host(Ud).tobytes(), st["iters"], st["normH2"], st["normU2"]))
    assert outs[0] == outs[1]
    Hr, Ur, sr = oracle.admm(M, S, H, U, tol=tol, max_iter=max_iter)
    if sr["iters"] == outs[0][2]:
        assert normwise(np.frombuffer(outs[0][0]).reshape(H.shape), Hr) <= TOL


@pytest.mark.parametrize("max_iter", [1, 17, 40])
def test_admm_iteration_chunking(B, max_iter):
    M, S, H, U = admm_inputs(2000, 32, 5)
    Hd, Ud = cu(H), cu(U)
    B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=max_iter)
    Hr, Ur, _ = oracle.admm(M, S, H, U, tol=0.0, max_iter=max_iter)
    assert normwise(host(Hd), Hr) <= TOL and normwise(host(Ud), Ur) <= TOL


def stop_margin(trace, j, eps):
    r, s, nH, nU = trace[j]
    return min(eps * nH - r, eps * nU - s) / (eps * (nH + nU))


@pytest.mark.parametrize("variant", [0, 1])
@pytest.mark.parametrize("eps,R", [(1e-1, 16), (1e-2, 32), (1e-3, 32), (1e-2, 64), (1e-2, 100)])
def test_admm_tolerance_mode(B, variant, eps, R):
    """Iteration count parity with the oracle's stopping rule (D3); U2 margin logged."""
    M, S, H, U = admm_inputs(3000, R, 99)
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=eps, max_iter=30, variant=variant)
    Hr, Ur, sr, tr = oracle.admm(M, S, H, U, tol=eps, max_iter=30, trace=True)
    if st["iters"] != sr["iters"]:
        j = min(st["iters"], sr["iters"]) - 1
        assert abs(stop_margin(tr, j, eps)) < 1e-12, "iteration counts differ away from a tie"
        pytest.skip("tie at the decisive iteration (U2)")
    assert normwise(host(Hd), Hr) <= TOL and normwise(host(Ud), Ur) <= TOL


def test_admm_identity_prox(B):
    M, S, H, U = admm_inputs(500, 16, 3)
    Hd, Ud = cu(H), cu(U)
    B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=12, prox=B.CSTF_PROX_IDENTITY)
    Hr, Ur, _ = oracle.admm(M, S, H, U, tol=0.0, max_iter=12, prox=oracle.PROX_IDENTITY)
    assert normwise(host(Hd), Hr) <= TOL
    assert np.any(host(Hd) < 0)


def test_admm_not_spd(B):
    R = 8
    with pytest.raises(B.CstfError) as e:
        B.cstf_admm_update(cu(np.ones((10, R))), cu(np.zeros((R, R))), cu(np.ones((10, R))), cu(np.zeros((10, R))),
                           tol=0.0, max_iter=3)
    assert e.value.status == B.CSTF_ERR_NOT_SPD


def run_both(B, dims, idx, vals, R, start, outer=10, tol=1e-2, max_iter=10, warm=0):
    ref = oracle.coalesce(dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=outer, tol=tol, max_iter=max_iter, warm=warm)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    opts = B.make_opts(R, outer_iters=outer, tol=tol, max_iter=max_iter, warm=warm)
    gpu = B.cstf_factorize(X, F, lam, opts)
    return orc, gpu, [host(f) for f in F], host(lam)


def test_factorize_planted_tiny(B):
    """configs[0]: fit after 10 outer iterations within 1e-6; every one of the 30 ADMM
    iteration counts equals the oracle's or differs at a tie (U2: |mu| < 1e-12 at the
    decisive pass -- the planted tensor is fitted exactly from outer iteration 6 on and
    its stop test then compares rounding noise, r, s, nU ~ 1e-31); factors <= 1e-6."""
    p = datagen.planted_tiny(1)
    start = datagen.perturbed_start(p, 1)
    orc, gpu, F, lam = run_both(B, p.dims, p.idx, p.vals, p.R, start)
    assert gpu["outer_done"] == 10
    n, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert n >= 15            # the first five outer iterations are decided well away from ties
    eq, ties = compare_all_iteration_counts(gpu["iters"], orc, 1e-2)
    assert eq + ties == 30 and eq >= 20, (eq, ties)
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    assert gpu["fit"][-1] >= 1 - 1e-6          # recovery (the 1e-8 gate is the oracle's pin P8)
    for a, b in zip(F, orc["factors"]):
        assert normwise(a, b) <= 1e-6
    assert normwise(lam, orc["lam"][-1]) <= 1e-6


@pytest.mark.parametrize("cfg,scale,R", [("nell2", 40, 16), ("enron", 40, 8), ("delicious", 2000, 8)])
def test_factorize_scaled_configs(B, cfg, scale, R):
    c = datagen.CONFIGS[cfg].scaled(scale, nnz_factor=scale * 20)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, R, c.seed)
    orc, gpu, F, lam = run_both(B, c.dims, idx, vals, R, start)
    n, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert tie is None, tie
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6


def test_factorize_fixed_iterations_protocol(B):
    """The timing protocol (eps = 0, 10 inner iterations) on a scaled NELL-2 shape."""
    c = datagen.CONFIGS["nell2"].scaled(20, nnz_factor=200)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, 32, c.seed)
    orc, gpu, F, lam = run_both(B, c.dims, idx, vals, 32, start, outer=3, tol=0.0)
    assert np.all(gpu["iters"] == 10)
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(a, b) <= 1e-6


@pytest.mark.parametrize("R,outer,tol,fit_tol,pinned,update,warm", [
    (8, 3, 1e-2, 0.0, False, 0, 0), (32, 4, 0.0, 0.0, True, 0, 0), (16, 3, 0.0, 1e-12, True, 0, 0),
    (5, 1, 0.0, 0.0, False, 0, 0), (16, 3, 0.0, 0.0, True, 1, 0), (32, 2, 0.0, 0.0, True, 2, 0),
    (32, 3, 0.0, 0.0, True, 0, 1), (8, 3, 1e-2, 0.0, False, 0, 1)])
def test_factorize_host_matches_device(B, R, outer, tol, fit_tol, pinned, update, warm):
    """The host-buffer path (factor copies overlapped with the computation: factor 0
    copied in during MTTKRP(0), each final factor copied out after its last update)
    gives the bits of the device path."""
    c = datagen.CONFIGS["enron"].scaled(60, nnz_factor=2000)
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    start = datagen.init_factors(c.dims, R, 1)
    opts = B.make_opts(R, outer_iters=outer, tol=tol, fit_tol=fit_tol, update=update, warm=warm)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    g1 = B.cstf_factorize(X, F, lam, opts)
    if pinned:
        hf = [torch.from_numpy(f.copy()).pin_memory() for f in start]
        hl = torch.zeros(R, dtype=torch.float64).pin_memory()
    else:
        hf = [f.copy() for f in start]
        hl = np.zeros(R)
    g2 = B.cstf_factorize_host(X, hf, hl, opts)
    assert np.array_equal(g1["fit"], g2["fit"])
    for a, b in zip(hf, F):
        assert np.array_equal(np.asarray(a), host(b))
    assert np.array_equal(np.asarray(hl), host(lam))


@pytest.mark.parametrize("R", [8, 32, 5, 64])
def test_mttkrp_kblocked_with_empty_blocks(B, R):
    """k-blocked copies (short output mode, long other mode): blocks of the long
    mode with no nonzeros still produce zero partial rows; rows absent from whole
    blocks, heavy rows and empty output rows all match the oracle."""
    rng = np.random.default_rng(R)
    nnz = 60000
    i = rng.integers(0, 40, nnz).astype(np.int32)
    i[i == 13] = 14                                   # output row 13 empty
    i[: nnz // 3] = 5                                 # a heavy output row
    j = rng.integers(0, 30, nnz).astype(np.int32)
    k = rng.integers(0, 2000, nnz).astype(np.int32)
    k[(k >= 256) & (k < 1024)] += 1000               # blocks 1..3 of mode 2 empty
    k = np.minimum(k, 1999).astype(np.int32)
    dims = (40, 30, 2000)
    vals = rng.random(nnz)
    X = B.cstf_tensor_load_coo(dims, [i, j, k], vals)
    ref = oracle.coalesce(dims, [i, j, k], vals)
    gi, gv = X.export_coo()
    assert np.array_equal(gv, ref.vals) and all(np.array_equal(a, b) for a, b in zip(gi, ref.idx))
    F = [rng.random((I, R)) for I in dims]
    Fd = [cu(f) for f in F]
    for n in range(3):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        assert normwise(host(M), oracle.mttkrp(ref, n, F)) <= TOL, n


@pytest.mark.parametrize("prox", [2, 3])
@pytest.mark.parametrize("R,variant", [(8, 0), (32, 0), (32, 1), (64, 0), (100, 0)])
def test_admm_l1_prox(B, prox, R, variant):
    """f3: L1 soft-threshold (and its non-negative form) in the fused kernel vs the oracle."""
    M, S, H, U = admm_inputs(1500, R, 7 + R)
    alpha = 0.2 * float(np.mean(np.diag(S)))
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=0.0, max_iter=10, prox=prox, alpha=alpha, variant=variant)
    Hr, Ur, sr = oracle.admm(M, S, H, U, tol=0.0, max_iter=10, prox=prox, alpha=alpha)
    assert normwise(host(Hd), Hr) <= TOL and normwise(host(Ud), Ur) <= TOL
    got = host(Hd)
    assert np.mean(got == 0.0) > 0.05                 # the threshold produces exact zeros
    if prox == 2:
        assert np.any(got < 0)


def test_factorize_nonneg_l1(B):
    c = datagen.CONFIGS["nell2"].scaled(40, nnz_factor=800)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, 16, c.seed)
    ref = oracle.coalesce(c.dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=5, tol=1e-2, max_iter=10, prox=oracle.PROX_NONNEG_L1, alpha=0.5)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(16))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(16, outer_iters=5, tol=1e-2, prox=3, alpha=0.5))
    n, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert tie is None
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6


@pytest.mark.parametrize("tol", [0.0, 1e-2])
@pytest.mark.parametrize("R,variant", [(8, 0), (32, 0), (32, 1), (64, 0), (100, 0)])
def test_admm_box_prox(B, R, variant, tol):
    """f3 (reading D25): the indicator of the box [0, alpha] in the fused kernel vs the
    oracle; alpha below the largest unconstrained value, so both bounds are active."""
    M, S, H, U = admm_inputs(1500, R, 11 + R)
    Hn, _, _ = oracle.admm(M, S, H, U, tol=0.0, max_iter=10)
    alpha = 0.5 * float(np.max(Hn))
    Hd, Ud = cu(H), cu(U)
    st = B.cstf_admm_update(cu(M), cu(S), Hd, Ud, tol=tol, max_iter=10, prox=B.CSTF_PROX_BOX, alpha=alpha,
                            variant=variant)
    Hr, Ur, sr = oracle.admm(M, S, H, U, tol=tol, max_iter=10, prox=oracle.PROX_BOX, alpha=alpha)
    assert st["iters"] == sr["iters"]
    assert normwise(host(Hd), Hr) <= TOL and normwise(host(Ud), Ur) <= TOL
    got = host(Hd)
    assert np.any(got == 0.0) and np.any(got == alpha) and got.max() <= alpha


def test_box_prox_rejects_nonpositive_bound(B):
    M, S, H, U = admm_inputs(100, 8, 3)
    with pytest.raises(B.CstfError):
        B.cstf_admm_update(cu(M), cu(S), cu(H), cu(U), prox=B.CSTF_PROX_BOX, alpha=0.0)


def test_factorize_box(B):
    """factorize with the box prox (alpha = 5, active: the oracle's fit differs from the
    plain non-negative run) against the oracle: counts, fits, factors."""
    c = datagen.CONFIGS["nell2"].scaled(40, nnz_factor=800)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, 16, c.seed)
    ref = oracle.coalesce(c.dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=5, tol=1e-2, max_iter=10, prox=oracle.PROX_BOX, alpha=5.0)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(16))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(16, outer_iters=5, tol=1e-2, prox=B.CSTF_PROX_BOX, alpha=5.0))
    n, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert tie is None
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(host(a), b) <= 1e-6


@pytest.mark.parametrize("update", ["hals", "mu"])
@pytest.mark.parametrize("I,R", [(1, 8), (1003, 8), (3001, 32), (999, 64), (300, 100)])
def test_hals_mu_updates(B, update, I, R):
    """f1: one HALS / MU update (3 sweeps) vs the oracle on positive data."""
    if update == "mu" and R > 64:
        pytest.skip("MU is built for R <= 64")
    M, S, H, U = admm_inputs(I, R, 5 + R)
    M = np.abs(M)
    Hd = cu(H)
    getattr(B, f"cstf_{update}_update")(cu(M), cu(S), Hd, sweeps=3)
    ref = getattr(oracle, update)(M, S, H, sweeps=3)
    assert normwise(host(Hd), ref) <= TOL
    assert np.min(host(Hd)) >= 0.0


@pytest.mark.parametrize("update,R", [(1, 16), (2, 16), (1, 40), (2, 40)])
def test_factorize_hals_mu(B, update, R):
    c = datagen.CONFIGS["enron"].scaled(60, nnz_factor=2000)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, R, c.seed)
    ref = oracle.coalesce(c.dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=5, max_iter=2, update=update)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    F = [cu(f) for f in start]
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=5, max_iter=2, update=update))
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(host(a), b) <= 1e-6


@pytest.mark.parametrize("R", [16, 32, 5])
def test_mttkrp_l2_blocked_copies(B, R, monkeypatch):
    """L2-blocked copies (virtual rows kb * I + i, fixed-order block reduction),
    forced at small sizes by shrinking the block to 64 rows."""
    monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "64")
    dims = (90, 2000, 700, 40)
    idx, vals = datagen.coo(dims, (2, 2, 3, 1), 120000, 21)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    gi, gv = X.export_coo()
    assert np.array_equal(gv, ref.vals) and all(np.array_equal(a, b) for a, b in zip(gi, ref.idx))
    F = datagen.init_factors(dims, R, 3)
    Fd = [cu(f) for f in F]
    for n in range(4):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        assert normwise(host(M), oracle.mttkrp(ref, n, F)) <= TOL, n
        monkeypatch.setenv("CSTF_L2_BATCH_BYTES", "1")        # one block per batch
        M1 = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M1)
        monkeypatch.delenv("CSTF_L2_BATCH_BYTES")
        assert normwise(host(M1), host(M)) <= TOL, n
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, Fd, lam, B.make_opts(R, outer_iters=3, tol=1e-2))
    orc = oracle.factorize(ref, F, outer_iters=3, tol=1e-2)
    n_, tie = compare_iteration_counts(gpu["iters"], orc, 1e-2)
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6


def test_mttkrp_l2_blocked_default(B, monkeypatch):
    """Default L2 blocking of short output modes against a factor that does not fit
    L2 (the Delicious mode-4 shape in small): layout chosen, parity with the oracle,
    bitwise repeatable under the dynamic chunk order, same result unblocked."""
    dims = (50, 600_000, 1000, 20)
    idx, vals = datagen.coo(dims, (1, 2, 3, 1), 1_500_000, 23)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    for n in (0, 2, 3):
        nblk, rows, bm = X.layout(n)
        assert bm == 1 and rows > 0 and nblk == -(-dims[1] // rows) and nblk > 1, (n, nblk, rows, bm)
    assert X.layout(1)[0] == 1
    R = 32
    F = datagen.init_factors(dims, R, 4)
    Fd = [cu(f) for f in F]
    monkeypatch.setenv("CSTF_L2_BLOCK", "0")
    Xp = B.cstf_tensor_load_coo(dims, idx, vals)
    assert all(Xp.layout(n)[0] == 1 for n in range(4))
    for n in range(4):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        first = host(M).copy()
        B.cstf_mttkrp(X, n, Fd, M)
        assert np.array_equal(host(M), first), n
        assert normwise(first, oracle.mttkrp(ref, n, F)) <= TOL, n
        Mp = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(Xp, n, Fd, Mp)
        assert normwise(first, host(Mp)) <= TOL, n


@pytest.mark.parametrize("R", [16, 32, 64])
def test_mttkrp_l2_blocked_long_rows_batches(B, R, monkeypatch):
    """Default L2 blocking of a long-row output mode (the Amazon case: >= 8 nonzeros per
    (row, block)); blocks processed in batches of any size (forced small budgets)
    match the oracle, and a fixed budget is bitwise repeatable."""
    dims = (20_000, 600_000, 30)
    idx, vals = datagen.coo(dims, (2, 2, 3), 5_000_000, 31)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    nblk, rows, bm = X.layout(0)
    assert bm == 1 and nblk == -(-dims[1] // rows) and nblk > 1
    ref = oracle.coalesce(dims, idx, vals)
    F = datagen.init_factors(dims, R, 6)
    Fd = [cu(f) for f in F]
    outs = []
    for budget in (None, 1, 3 * dims[0] * R * 8):
        if budget is None:
            monkeypatch.delenv("CSTF_L2_BATCH_BYTES", raising=False)
        else:
            monkeypatch.setenv("CSTF_L2_BATCH_BYTES", str(budget))
        M = cu(np.full((dims[0], R), np.nan))
        B.cstf_mttkrp(X, 0, Fd, M)
        outs.append(host(M).copy())
        B.cstf_mttkrp(X, 0, Fd, M)
        assert np.array_equal(host(M), outs[-1])
    want = oracle.mttkrp(ref, 0, F)
    for o in outs:
        assert normwise(o, want) <= TOL
    # one launch per block with a persisting L2 window on its slab (forced at this size)
    monkeypatch.delenv("CSTF_L2_BATCH_BYTES", raising=False)
    monkeypatch.setenv("CSTF_L2_PERSIST", str(32 << 20))
    M = cu(np.full((dims[0], R), np.nan))
    B.cstf_mttkrp(X, 0, Fd, M)
    first = host(M).copy()
    B.cstf_mttkrp(X, 0, Fd, M)
    assert np.array_equal(host(M), first) and normwise(first, want) <= TOL


@pytest.mark.parametrize("budget", [None, "1"])
def test_mttkrp_l2_blocked_empty_blocks(B, budget, monkeypatch):
    """Forced L2 blocks where most blocks of the blocked factor hold no nonzeros (and
    rows of the output mode without nonzeros), whole-batch and one-block batches."""
    monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "64")
    if budget:
        monkeypatch.setenv("CSTF_L2_BATCH_BYTES", budget)
    dims = (50, 3000, 20)
    idx, vals = datagen.coo(dims, (2, 2, 1), 40000, 41)
    j = idx[1].astype(np.int64)
    idx[1] = np.where(j < 1500, j % 500, 2500 + j % 500).astype(np.int32)   # blocks 8..38 empty
    idx[0] = (idx[0] // 2 * 2).astype(np.int32)                              # odd rows empty
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    assert X.layout(0)[0] > 1
    ref = oracle.coalesce(dims, idx, vals)
    F = datagen.init_factors(dims, 16, 8)
    Fd = [cu(f) for f in F]
    M = cu(np.full((dims[0], 16), np.nan))
    B.cstf_mttkrp(X, 0, Fd, M)
    got = host(M)
    assert normwise(got, oracle.mttkrp(ref, 0, F)) <= TOL
    assert np.all(got[1::2] == 0.0)


def test_factorize_bitwise_deterministic(B):
    """Fixed grids and fixed reduction orders everywhere: two runs are bit-identical."""
    c = datagen.CONFIGS["enron"].scaled(60, nnz_factor=1000)
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    start = datagen.init_factors(c.dims, 16, 2)
    outs = []
    for _ in range(2):
        F = [cu(f) for f in start]
        lam = cu(np.zeros(16))
        rep = B.cstf_factorize(X, F, lam, B.make_opts(16, outer_iters=4, tol=1e-2))
        outs.append((rep["fit"].tobytes(), rep["iters"].tobytes(), b"".join(host(f).tobytes() for f in F)))
    assert outs[0] == outs[1]


def test_eight_mode_tensor(B):
    """N = 8 (7 other modes: 48-byte records, generic MTTKRP path) end to end."""
    dims = (5, 4, 6, 3, 7, 4, 5, 3)
    idx, vals = datagen.coo(dims, (1, 2, 1, 1, 2, 1, 1, 1), 4000, 31)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    assert X.info()["hash"] == ref.hash
    R = 4
    F = datagen.init_factors(dims, R, 5)
    for n in (0, 7):
        M = cu(np.zeros((dims[n], R)))
        B.cstf_mttkrp(X, n, [cu(f) for f in F], M)
        assert normwise(host(M), oracle.mttkrp(ref, n, F)) <= TOL
    Fd = [cu(f) for f in F]
    lam = cu(np.zeros(R))
    gpu = B.cstf_factorize(X, Fd, lam, B.make_opts(R, outer_iters=3, tol=1e-2))
    orc = oracle.factorize(ref, F, outer_iters=3, tol=1e-2)
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6


def test_dead_column_and_rank_one(B):
    """A component that dies (zero column, lambda = 0, reading D8) stays zero without NaN;
    R = 1 runs the generic widths."""
    c = datagen.CONFIGS["nell2"].scaled(100, nnz_factor=5000)
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    ref = oracle.coalesce(c.dims, idx, vals)
    for R in (1, 6):
        F = datagen.init_factors(c.dims, R, 8)
        if R > 1:
            for f in F:
                f[:, 2] = 0.0                      # component 2 is dead from the start
        Fd = [cu(f) for f in F]
        lam = cu(np.zeros(R))
        gpu = B.cstf_factorize(X, Fd, lam, B.make_opts(R, outer_iters=3, tol=1e-2))
        orc = oracle.factorize(ref, F, outer_iters=3, tol=1e-2)
        assert np.all(np.isfinite(gpu["fit"]))
        assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
        if R > 1:
            assert host(lam)[2] == 0.0 and all(np.all(host(f)[:, 2] == 0.0) for f in Fd)


def test_nonfinite_input_is_reported(B):
    dims = (20, 15, 10)
    idx, vals = datagen.coo(dims, (1, 1, 1), 500, 4)
    vals = vals.copy()
    vals[7] = np.inf
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    F = [cu(f) for f in datagen.init_factors(dims, 4, 1)]
    with pytest.raises(B.CstfError) as e:
        B.cstf_factorize(X, F, cu(np.zeros(4)), B.make_opts(4, outer_iters=2, tol=1e-2))
    assert e.value.status in (B.CSTF_ERR_NUMERIC, B.CSTF_ERR_NOT_SPD)


@pytest.mark.parametrize("R", [32, 16, 8, 64, 5])
@pytest.mark.parametrize("window", ["1", "0"])
def test_mttkrp_hot_row_tables(B, R, window, monkeypatch):
    """Hot-row tables: records of the rows with the most nonzeros
    point into a separate table refreshed from the factor and read under a persisting
    L2 window.  Forced at small size (CSTF_HOT_ROWS): MTTKRP of every mode against the
    oracle (fast kernels for R = 16/32/64, generic otherwise), with and without the
    window, the export restores the canonical COO bit for bit, and the result is
    bitwise the one of the store without hot rows."""
    monkeypatch.setenv("CSTF_HOT_ROWS", "300")
    monkeypatch.setenv("CSTF_HOT_WINDOW", window)
    monkeypatch.setenv("CSTF_MTTKRP_G", "0")           # the same lane-group width with and without hot rows
    dims = (90, 5000, 1200, 40)
    idx, vals = datagen.coo(dims, (2, 2, 3, 1), 200_000, 51)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    gi, gv = X.export_coo()
    assert np.array_equal(gv, ref.vals) and all(np.array_equal(a, b) for a, b in zip(gi, ref.idx))
    monkeypatch.setenv("CSTF_HOT", "0")
    Xp = B.cstf_tensor_load_coo(dims, idx, vals)
    F = datagen.init_factors(dims, R, 9)
    Fd = [cu(f) for f in F]
    for n in range(4):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        got = host(M).copy()
        assert normwise(got, oracle.mttkrp(ref, n, F)) <= TOL, n
        Mp = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(Xp, n, Fd, Mp)
        if R in (16, 32, 64):          # same fast kernel and order (other R: generic vs fast kernel)
            assert np.array_equal(got, host(Mp)), n
        else:
            assert normwise(got, host(Mp)) <= TOL, n
    # a changed factor is picked up (standalone calls refresh the tables)
    F2 = [f * 1.5 for f in F]
    M = cu(np.full((dims[0], R), np.nan))
    B.cstf_mttkrp(X, 0, [cu(f) for f in F2], M)
    assert normwise(host(M), oracle.mttkrp(ref, 0, F2)) <= TOL


@pytest.mark.parametrize("unr", ["1", "2", "3", "4"])
def test_mttkrp_hot_unrolled_gathers(B, unr, monkeypatch):
    """Hot-row copies at R = 32 issue the row loads of several steps before the first
    product (mttkrp_unr: 2 steps for short rows, 4 for medium ones).  Forced hot rows,
    one mode per row class (long 3333 / short 10 / medium 37 / long 7500 nonzeros per
    row): every unroll depth matches the oracle, and -- the per-group accumulation
    order is unchanged -- is bitwise equal to the one-step kernel."""
    monkeypatch.setenv("CSTF_HOT_ROWS", "400")
    dims = (90, 30000, 8000, 40)
    idx, vals = datagen.coo(dims, (2, 2, 3, 1), 300_000, 52)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    ref = oracle.coalesce(dims, idx, vals)
    F = datagen.init_factors(dims, 32, 10)
    Fd = [cu(f) for f in F]
    for n in range(4):
        monkeypatch.setenv("CSTF_MTTKRP_UNR", "1")
        M1 = cu(np.full((dims[n], 32), np.nan))
        B.cstf_mttkrp(X, n, Fd, M1)
        monkeypatch.setenv("CSTF_MTTKRP_UNR", unr)
        M = cu(np.full((dims[n], 32), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        got = host(M).copy()
        assert normwise(got, oracle.mttkrp(ref, n, F)) <= TOL, n
        assert np.array_equal(got, host(M1)), n


@pytest.mark.parametrize("tol,R", [(1e-2, 16), (0.0, 32)])
def test_factorize_hot_row_tables(B, tol, R, monkeypatch):
    """factorize keeps the hot-row tables current after every update (forced hot rows)."""
    monkeypatch.setenv("CSTF_HOT_ROWS", "200")
    c = datagen.CONFIGS["delicious"].scaled(1000, nnz_factor=700)
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, R, c.seed)
    orc, gpu, F, lam = run_both(B, c.dims, idx, vals, R, start, outer=4, tol=tol)
    n, tie = compare_iteration_counts(gpu["iters"], orc, tol if tol > 0 else 1e-2)
    assert tie is None
    assert np.max(np.abs(gpu["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(F, orc["factors"]):
        assert normwise(a, b) <= 1e-6
