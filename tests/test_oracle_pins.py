"""Pins of the FP64 oracle (oracle/) to things other than itself (CPU only).

Each test names the pin from DESIGN.md "Oracle pins"
and the paper passage it anchors.  None of them re-types the oracle's formula:
they use dense definitions (matricisation x explicit Khatri-Rao), brute force
(active-set NNLS, dictionary coalescing), closed forms (least squares, KKT),
identities of the iteration itself (dual update => primal residual), spectral
bounds, and planted exact recovery.
"""
import json
import os
import subprocess
import sys
from itertools import combinations

import numpy as np
import pytest

import datagen
import oracle

HERE = os.path.dirname(os.path.abspath(__file__))


def normwise(a, b):
    """Reading D18: max|a-b| / max|b|."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    den = np.max(np.abs(b))
    return float(np.max(np.abs(a - b)) / (den if den > 0 else 1.0))


def random_coo(rng, dims, nnz, dup_frac=0.2, neg=True, zeros=True):
    idx = [rng.integers(0, I, nnz).astype(np.int32) for I in dims]
    ndup = int(nnz * dup_frac)
    if ndup:
        src = rng.integers(0, nnz, ndup)
        dst = rng.integers(0, nnz, ndup)
        for a in idx:
            a[dst] = a[src]
    vals = rng.random(nnz) + 0.1
    if neg:
        vals[rng.random(nnz) < 0.1] *= -1
    if zeros:
        vals[rng.random(nnz) < 0.05] = 0.0
    return idx, vals


def dense_of(X):
    D = np.zeros(X.dims)
    D[tuple(X.idx)] = X.vals        # canonical: indices unique
    return D


def unfold(D, n):
    """Mode-n matricisation X_(n): rows i_n, columns the other
    indices in increasing mode order, last fastest (one self-consistent pairing, D16)."""
    return np.moveaxis(D, n, 0).reshape(D.shape[n], -1)


def khatri_rao_except(factors, n):
    """Explicit Khatri-Rao of the other factors, row order
    matching `unfold` (first other mode slowest)."""
    R = factors[0].shape[1]
    kr = None
    for k, F in enumerate(factors):
        if k == n:
            continue
        kr = F.copy() if kr is None else (kr[:, None, :] * F[None, :, :]).reshape(-1, R)
    return kr


# --------------------------------------------------------------------- O1 coalesce
def test_coalesce_bruteforce(rng):
    """O1 vs a dictionary sum in input order (bit-exact), sorted keys, ||X||^2."""
    dims = (7, 5, 6, 3)
    idx, vals = random_coo(rng, dims, 400, dup_frac=0.4)
    X = oracle.coalesce(dims, idx, vals)
    acc = {}
    for p in range(len(vals)):
        key = tuple(int(a[p]) for a in idx)
        acc[key] = acc[key] + vals[p] if key in acc else vals[p]
    keys = sorted(acc)
    assert X.nnz == len(keys)
    got = list(zip(*[a.tolist() for a in X.idx]))
    assert got == keys
    assert np.array_equal(X.vals, np.array([acc[k] for k in keys]))     # bit-exact
    assert X.normX2 == pytest.approx(float(np.sum(X.vals ** 2)), rel=1e-14)


def test_coalesce_hash_order_invariant(rng):
    """The canonical checksum depends on the tensor, not on the input order."""
    dims = (9, 4, 11)
    cells = rng.choice(int(np.prod(dims)), 300, replace=False)     # distinct cells
    idx = [a.astype(np.int32) for a in np.unravel_index(cells, dims)]
    vals = rng.random(300)
    perm = rng.permutation(300)
    X1 = oracle.coalesce(dims, idx, vals)
    X2 = oracle.coalesce(dims, [a[perm] for a in idx], vals[perm])
    assert X1.hash == X2.hash
    assert oracle.canonical_hash(X1.idx, X1.vals) == X1.hash
    v = X1.vals.copy(); v[17] = np.nextafter(v[17], np.inf)
    assert oracle.canonical_hash(X1.idx, v) != X1.hash


def test_coalesce_rejects_out_of_range():
    with pytest.raises(oracle.OracleError):
        oracle.coalesce((3, 3), [np.array([0, 3], np.int32), np.array([0, 1], np.int32)], np.ones(2))


def test_coalesce_empty():
    X = oracle.coalesce((3, 4, 5), [np.zeros(0, np.int32)] * 3, np.zeros(0))
    assert X.nnz == 0 and X.normX2 == 0.0


# --------------------------------------------------------------------- P1 MTTKRP
@pytest.mark.parametrize("dims", [(8, 6, 7), (5, 4, 6, 3), (9, 7)])
@pytest.mark.parametrize("R", [1, 5, 8])
def test_P1_mttkrp_dense_khatri_rao(rng, dims, R):
    """P1: sparse MTTKRP (Fig. 2) == X_(n) (KR of the others) (L386-387)."""
    idx, vals = random_coo(rng, dims, int(0.4 * np.prod(dims)))
    X = oracle.coalesce(dims, idx, vals)
    F = [rng.random((I, R)) for I in dims]
    D = dense_of(X)
    for n in range(len(dims)):
        ref = unfold(D, n) @ khatri_rao_except(F, n)
        got = oracle.mttkrp(X, n, F)
        assert normwise(got, ref) <= 1e-13
        rows = np.array([0, dims[n] - 1, dims[n] // 2, 0])
        assert np.array_equal(oracle.mttkrp_rows(X, n, F, rows), got[rows])


def test_P1_mttkrp_empty_rows_are_zero(rng):
    dims = (10, 4, 4)
    idx = [np.array([2, 2, 7], np.int32), np.array([0, 1, 3], np.int32), np.array([1, 1, 2], np.int32)]
    X = oracle.coalesce(dims, idx, np.array([1.0, 2.0, 3.0]))
    F = [rng.random((I, 3)) for I in dims]
    M = oracle.mttkrp(X, 0, F)
    assert np.all(M[[0, 1, 3, 4, 5, 6, 8, 9]] == 0.0)
    assert normwise(M, unfold(dense_of(X), 0) @ khatri_rao_except(F, 0)) <= 1e-15


# --------------------------------------------------------------------- Gram / Hadamard / Cholesky
def test_gram_matches_blas(rng):
    """O3 vs the library product H^T H (a plain textbook/library routine)."""
    H = rng.random((10_000, 7))
    assert normwise(oracle.gram(H), H.T @ H) <= 1e-13
    G = oracle.gram(H)
    assert np.array_equal(G, G.T)


def test_hadamard_except_definition(rng):
    """O4: S = *_{k!=n} G^(k); for N=2 it is the other Gram itself (L494)."""
    Gs = [rng.random((4, 4)) for _ in range(3)]
    assert np.array_equal(oracle.hadamard_except(Gs[:2], 0), Gs[1])
    S = oracle.hadamard_except(Gs, 1)
    assert normwise(S, Gs[0] * Gs[2]) == 0.0


def test_cholesky_library_special_case(rng):
    """O6 vs numpy.linalg.cholesky, and L L^T reconstructs A."""
    B = rng.random((12, 12))
    A = B @ B.T + 12 * np.eye(12)
    L = oracle.cholesky(A)
    assert normwise(L, np.linalg.cholesky(A)) <= 1e-14
    assert normwise(L @ L.T, A) <= 1e-14
    assert np.all(np.triu(L, 1) == 0)


def test_cholesky_not_spd():
    with pytest.raises(oracle.OracleError) as e:
        oracle.cholesky(np.array([[1.0, 2.0], [2.0, 1.0]]))
    assert e.value.code == oracle.NOT_SPD


def make_S(rng, R, nmodes=3, rows=50):
    """S as the method builds it: Hadamard of Grams of non-negative factors."""
    Gs = [oracle.gram(rng.random((rows, R))) for _ in range(nmodes)]
    return oracle.hadamard_except(Gs, 0)


# --------------------------------------------------------------------- P2 brute-force NNLS
def nnls_bruteforce(S, m):
    """min_h 1/2 h^T S h - m^T h, h >= 0, by enumerating passive sets (R <= 4)."""
    R = len(m)
    best, best_h = np.inf, None
    for k in range(R + 1):
        for P in combinations(range(R), k):
            h = np.zeros(R)
            if P:
                P = list(P)
                h[P] = np.linalg.solve(S[np.ix_(P, P)], m[P])
                if np.any(h < 0):
                    continue
            f = 0.5 * h @ S @ h - m @ h
            if f < best:
                best, best_h = f, h
    return best_h


@pytest.mark.parametrize("R", [2, 3, 4])
def test_P2_admm_fixed_point_is_nnls(rng, R):
    """P2: ADMM (eps=0, many iterations) == brute-force active-set NNLS per row."""
    S = make_S(rng, R)
    I = 40
    M = (rng.random((I, R)) - 0.45) * np.diag(S).mean()      # mixed signs => active constraints
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=5000)
    ref = np.array([nnls_bruteforce(S, M[i]) for i in range(I)])
    assert np.any(ref == 0.0) and np.any(ref > 0)
    assert normwise(H, ref) <= 1e-10
    assert st["iters"] == 5000


# --------------------------------------------------------------------- P3 closed form
def test_P3_positive_least_squares_solution_recovered(rng):
    """P3: M = H* S with H* > 0 => the unconstrained LS solution is feasible => ADMM -> H*."""
    R, I = 8, 300
    S = make_S(rng, R)
    Hs = rng.random((I, R)) + 0.1
    M = Hs @ S
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=3000)
    assert normwise(H, Hs) <= 1e-10
    assert np.max(np.abs(U)) <= 1e-10 * np.max(np.abs(M))


# --------------------------------------------------------------------- P4 KKT
def test_P4_kkt_complementarity(rng):
    """P4: at the fixed point H = H~, so rho U = H S - M, U >= 0, H >= 0, H o U = 0."""
    R, I = 6, 200
    S = make_S(rng, R)
    M = (rng.random((I, R)) - 0.4) * np.diag(S).mean()
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=4000)
    rho = st["rho"]
    scale = np.max(np.abs(M))
    assert np.max(np.abs(rho * U - (H @ S - M))) <= 1e-10 * scale
    assert np.min(H) >= 0.0
    assert np.min(U) >= -1e-12 * scale / rho
    assert np.max(np.abs(H * U)) <= 1e-10 * scale * np.max(H) / rho


# --------------------------------------------------------------------- stopping rule (D3)
def test_D3_residuals_follow_from_the_iteration(rng):
    """The four sums of pass j are properties of the iterates: the dual update
    U_j - U_{j-1} = H_j - H~_j gives r_j; s_j = ||H_j - H_{j-1}||^2; nH, nU the
    norms of the updated iterates.  The stop count is the first j with
    r_j < eps nH_j and s_j < eps nU_j (reading D3)."""
    R, I = 5, 120
    S = make_S(rng, R)
    M = (rng.random((I, R)) - 0.3) * np.diag(S).mean()
    H0 = rng.random((I, R)); U0 = np.zeros((I, R))
    Hs, Us = [H0], [U0]
    for j in range(1, 9):
        H, U, _ = oracle.admm(M, S, H0, U0, tol=0.0, max_iter=j)
        Hs.append(H); Us.append(U)
    _, _, _, tr = oracle.admm(M, S, H0, U0, tol=0.0, max_iter=8, trace=True)
    for j in range(1, 9):
        r = np.sum((Us[j] - Us[j - 1]) ** 2)
        s = np.sum((Hs[j] - Hs[j - 1]) ** 2)
        assert tr[j - 1, 0] == pytest.approx(r, rel=1e-9, abs=1e-300)
        assert tr[j - 1, 1] == pytest.approx(s, rel=1e-9, abs=1e-300)
        assert tr[j - 1, 2] == pytest.approx(np.sum(Hs[j] ** 2), rel=1e-12)
        assert tr[j - 1, 3] == pytest.approx(np.sum(Us[j] ** 2), rel=1e-12)
    for eps in (1e-1, 1e-2, 1e-3):
        want = next((j for j in range(1, 9) if tr[j - 1, 0] < eps * tr[j - 1, 2]
                     and tr[j - 1, 1] < eps * tr[j - 1, 3]), 8)
        _, _, st = oracle.admm(M, S, H0, U0, tol=eps, max_iter=8)
        assert st["iters"] == want


def test_D3_zero_dual_norm_means_continue(rng):
    """nU = 0 can never satisfy s < eps*nU: with U staying 0 the loop runs max_iter."""
    R, I = 4, 50
    S = make_S(rng, R)
    Hs = rng.random((I, R)) + 0.5
    M = Hs @ S
    _, _, st = oracle.admm(M, S, Hs, np.zeros((I, R)), tol=1e-1, max_iter=7)
    assert st["normU2"] <= 1e-20 and st["iters"] == 7


# --------------------------------------------------------------------- P5 / P6
@pytest.mark.parametrize("R", [4, 8, 16])
def test_P5_conditioning_bound(rng, R):
    """P5: S PSD (Schur product theorem) => kappa(S + rho I) <= R + 1 with rho = tr(S)/R."""
    for _ in range(5):
        S = make_S(rng, R)
        _, _, st = oracle.admm(np.zeros((1, R)), S, np.zeros((1, R)), np.zeros((1, R)), max_iter=1)
        assert st["rho"] == pytest.approx(np.trace(S) / R, rel=1e-15)
        ev = np.linalg.eigvalsh(S + st["rho"] * np.eye(R))
        assert ev[-1] / ev[0] <= R + 1 + 1e-9


def test_P6_rho_is_one_for_normalised_factors(rng):
    """P6: normalised factors have unit Gram diagonals, so tr(S) = R and rho = 1."""
    R = 8
    Fs = [oracle.normalize(rng.random((I, R)))[0] for I in (30, 40, 50)]
    for F in Fs:
        assert np.allclose(np.linalg.norm(F, axis=0), 1.0, rtol=0, atol=1e-15)
    Gs = [oracle.gram(F) for F in Fs]
    S = oracle.hadamard_except(Gs, 2)
    _, _, st = oracle.admm(np.zeros((1, R)), S, np.zeros((1, R)), np.zeros((1, R)), max_iter=1)
    assert abs(st["rho"] - 1.0) <= 1e-15


def test_normalize_reconstructs_and_zero_column(rng):
    """O8 / D8: H = Hn diag(lam); a zero column stays zero with lam = 0."""
    H = rng.random((100, 5)); H[:, 3] = 0.0
    Hn, lam = oracle.normalize(H)
    assert lam[3] == 0.0 and np.all(Hn[:, 3] == 0.0)
    assert normwise(Hn * lam, H) <= 1e-15
    assert normwise(lam, np.linalg.norm(H, axis=0)) <= 1e-15


# --------------------------------------------------------------------- P7 fit
def test_P7_fit_inner_product_equals_dense(rng):
    """P7: inner-product fit (D12) == 1 - ||X - [[lam; H]]||_F / ||X|| evaluated densely."""
    dims = (9, 8, 7)
    R = 4
    idx, vals = random_coo(rng, dims, 250, neg=False, zeros=False)
    X = oracle.coalesce(dims, idx, vals)
    Hs, lams = [], []
    for I in dims:
        Hn, lam = oracle.normalize(rng.random((I, R)))
        Hs.append(Hn); lams.append(lam)
    lam = lams[-1] * 3.0
    M = oracle.mttkrp(X, len(dims) - 1, Hs)
    f = oracle.fit(X.normX2, M, Hs[-1], lam, [oracle.gram(H) for H in Hs])
    Xhat = np.einsum("r,ir,jr,kr->ijk", lam, *Hs)
    ref = 1 - np.linalg.norm(dense_of(X) - Xhat) / np.linalg.norm(dense_of(X))
    assert f == pytest.approx(ref, abs=1e-13)


# --------------------------------------------------------------------- P8 planted recovery
def test_P8_planted_exact_recovery_pins_warm_start():
    """P8: configs[0] planted rank-8 tensor, truth + 5% start, eps=1e-2, max_iter=10.
    Reading D4 (scaled warm start) reaches fit >= 1 - 1e-8 in 10 outer iterations;
    the literal reading (normalised warm start) plateaus below it."""
    p = datagen.planted_tiny(1)
    X = oracle.coalesce(p.dims, p.idx, p.vals)
    assert X.nnz == 2000
    start = datagen.perturbed_start(p, 1)
    res = oracle.factorize(X, start, outer_iters=10, tol=1e-2, max_iter=10, warm=oracle.WARM_SCALED)
    assert res["fit"][-1] >= 1 - 1e-8
    assert np.all(res["iters"] >= 1) and np.all(res["iters"] <= 10)
    assert np.any(res["iters"] < 10)                       # early termination occurs
    lit = oracle.factorize(X, start, outer_iters=10, tol=1e-2, max_iter=10, warm=oracle.WARM_NORMALIZED)
    assert lit["fit"][-1] < 1 - 1e-5
    # recovered model reproduces the planted tensor cell by cell
    H = res["factors"]
    lam = res["lam"][-1]
    Xhat = np.einsum("r,ir,jr,kr->ijk", lam, *H)
    D = dense_of(X)
    assert np.max(np.abs(Xhat - D)) <= 1e-4 * np.max(D)


# --------------------------------------------------------------------- P9 cost model
def test_P9_paper_cost_model_values():
    """P9: Eq. 5 reproduces the printed AI 0.29 / 0.47 / 0.83 (L683-684) and the
    fusion count 4IR+2IR -> 3IR+IR, ~33% (L823-829)."""
    from paper_conf_icpp_sohksc24_b200 import costmodel as cm
    g = json.load(open(os.path.join(HERE, "golden", "paper_cost_model.json")))
    for R, printed in g["printed_ai"].items():
        R = int(R)
        # the paper prints 2 decimals (0.8352 appears as 0.83: truncated, not rounded)
        for ai in (cm.paper_ai_limit(R), cm.paper_ai(10 ** 7, R)):
            assert printed in (round(ai, 2), np.floor(ai * 100) / 100)
    f = g["fusion_compute_auxiliary"]
    r0, w0 = cm.fusion_compute_auxiliary_words(1, 1, fused=False)
    r1, w1 = cm.fusion_compute_auxiliary_words(1, 1, fused=True)
    assert (r0, w0, r1, w1) == (f["unfused_reads_IR"], f["unfused_writes_IR"],
                                f["fused_reads_IR"], f["fused_writes_IR"])
    assert abs(1 - (r1 + w1) / (r0 + w0) - 1 / 3) < 1e-12


# --------------------------------------------------------------------- P10 unconstrained
def test_P10_identity_prox_gives_cp_als_update(rng):
    """P10: with the identity prox ADMM converges to M S^-1, the CP-ALS update (L360-368)."""
    R, I = 6, 80
    S = make_S(rng, R)
    M = rng.random((I, R)) - 0.5
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=3000,
                           prox=oracle.PROX_IDENTITY)
    assert normwise(H, np.linalg.solve(S, M.T).T) <= 1e-10


# --------------------------------------------------------------------- P11 determinism
def test_P11_thread_count_determinism():
    code = (
        "import numpy as np, datagen, oracle, hashlib;"
        "cfg = datagen.Config('t', (3000, 2000, 5000), (2, 2, 3), 200000, 8, 7);"
        "idx, v = cfg.generate(); X = oracle.coalesce(cfg.dims, idx, v);"
        "F = datagen.init_factors(cfg.dims, 8, 7);"
        "r = oracle.factorize(X, F, outer_iters=2, tol=1e-2, max_iter=10);"
        "h = hashlib.sha256(); [h.update(f.tobytes()) for f in r['factors']];"
        "h.update(r['fit'].tobytes()); h.update(r['iters'].tobytes()); print(h.hexdigest())"
    )
    out = []
    for th in ("1", "3", "8"):
        env = dict(os.environ, OMP_NUM_THREADS=th, PYTHONPATH=os.path.dirname(HERE))
        out.append(subprocess.check_output([sys.executable, "-c", code], env=env).strip())
    assert out[0] == out[1] == out[2]


# --------------------------------------------------------------------- f3: L1 proximity operators
def lasso_bruteforce(S, m, alpha, nonneg):
    """min_h 1/2 h^T S h - m^T h + alpha ||h||_1 (h >= 0 if nonneg) by enumerating
    sign patterns (each coordinate -, 0, +): on a fixed pattern the problem is an
    equality-constrained quadratic with the linear term shifted by alpha*sign."""
    from itertools import product
    R = len(m)
    best, best_h = np.inf, None
    signs = (0, 1) if nonneg else (-1, 0, 1)
    for pat in product(signs, repeat=R):
        P = [i for i in range(R) if pat[i] != 0]
        h = np.zeros(R)
        if P:
            sg = np.array([pat[i] for i in P], dtype=float)
            h[P] = np.linalg.solve(S[np.ix_(P, P)], m[P] - alpha * sg)
            if np.any(np.sign(h[P]) != sg):
                continue
        f = 0.5 * h @ S @ h - m @ h + alpha * np.abs(h).sum()
        if f < best:
            best, best_h = f, h
    return best_h


@pytest.mark.parametrize("prox,nonneg", [(oracle.PROX_L1, False), (oracle.PROX_NONNEG_L1, True)])
@pytest.mark.parametrize("R", [2, 3])
def test_f3_l1_prox_fixed_point_is_lasso(rng, prox, nonneg, R):
    """ADMM with r = alpha ||.||_1 (+ R_+) converges to the brute-force (non-negative) lasso."""
    S = make_S(rng, R)
    I = 30
    M = (rng.random((I, R)) - 0.4) * np.diag(S).mean()
    alpha = 0.3 * np.diag(S).mean()
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=6000, prox=prox, alpha=alpha)
    ref = np.array([lasso_bruteforce(S, M[i], alpha, nonneg) for i in range(I)])
    assert np.any(ref == 0.0)
    assert normwise(H, ref) <= 1e-9


def test_f3_l1_with_zero_alpha_is_the_plain_operator(rng):
    R, I = 5, 40
    S = make_S(rng, R)
    M = rng.random((I, R)) - 0.5
    a = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), max_iter=20, prox=oracle.PROX_NONNEG_L1, alpha=0.0)
    b = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), max_iter=20, prox=oracle.PROX_NONNEG)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


def box_bruteforce(S, m, hi):
    """min_h 1/2 h^T S h - m^T h over the box 0 <= h <= hi (S SPD), by enumerating for
    every coordinate the state lower bound / free / upper bound (3^R patterns) and
    keeping the feasible stationary point of least objective."""
    from itertools import product
    R = len(m)
    best, best_h = np.inf, None
    for pat in product((0, 1, 2), repeat=R):
        h = np.where(np.array(pat) == 2, hi, 0.0)
        F = [i for i in range(R) if pat[i] == 1]
        if F:
            C = [i for i in range(R) if pat[i] != 1]
            rhs = m[F] - (S[np.ix_(F, C)] @ h[C] if C else 0.0)
            h[F] = np.linalg.solve(S[np.ix_(F, F)], rhs)
            if np.any(h[F] < 0.0) or np.any(h[F] > hi):
                continue
        f = 0.5 * h @ S @ h - m @ h
        if f < best:
            best, best_h = f, h
    return best_h


@pytest.mark.parametrize("R", [2, 3])
def test_f3_box_fixed_point_is_bruteforce_qp(rng, R):
    """Reading D25: ADMM with the indicator of [0, alpha] converges to the box-constrained
    least-squares minimiser found by brute force; both bounds are active somewhere."""
    S = make_S(rng, R)
    I = 40
    M = (rng.random((I, R)) - 0.3) * 2.0 * np.diag(S).mean()
    hi = 0.6
    H, U, st = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), tol=0.0, max_iter=6000,
                           prox=oracle.PROX_BOX, alpha=hi)
    ref = np.array([box_bruteforce(S, M[i], hi) for i in range(I)])
    assert np.any(ref == 0.0) and np.any(ref == hi)
    assert normwise(H, ref) <= 1e-9


def test_f3_box_with_unreachable_bound_is_the_plain_operator(rng):
    """A box whose upper bound is never reached runs exactly the non-negativity operator."""
    R, I = 5, 40
    S = make_S(rng, R)
    M = rng.random((I, R)) - 0.5
    a = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), max_iter=20, prox=oracle.PROX_BOX, alpha=1e300)
    b = oracle.admm(M, S, np.zeros((I, R)), np.zeros((I, R)), max_iter=20, prox=oracle.PROX_NONNEG)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


# --------------------------------------------------------------------- f1: HALS / MU
def nnls_objective(S, M, H):
    return float(np.sum(0.5 * np.einsum("ir,rs,is->i", H, S, H) - np.einsum("ir,ir->i", M, H)))


@pytest.mark.parametrize("R", [2, 3, 4])
def test_f1_hals_converges_to_nnls(rng, R):
    """HALS is exact coordinate descent on the per-row NNLS: it reaches the brute-force minimiser."""
    S = make_S(rng, R)
    I = 40
    M = (rng.random((I, R)) - 0.45) * np.diag(S).mean()
    H = oracle.hals(M, S, np.zeros((I, R)) + 0.1, sweeps=3000)
    ref = np.array([nnls_bruteforce(S, M[i]) for i in range(I)])
    assert normwise(H, ref) <= 1e-9


@pytest.mark.parametrize("update", ["hals", "mu"])
def test_f1_monotone_objective(rng, update):
    """Both schemes never increase the NNLS objective (Lee-Seung for MU; exact
    coordinate minimisation for HALS) on non-negative data."""
    R, I = 6, 200
    S = make_S(rng, R)
    M = rng.random((I, R)) * np.diag(S).mean()
    H = rng.random((I, R))
    f = getattr(oracle, update)
    prev = nnls_objective(S, M, H)
    for _ in range(30):
        H = f(M, S, H, sweeps=1)
        cur = nnls_objective(S, M, H)
        assert cur <= prev + 1e-12 * abs(prev)
        prev = cur
    assert np.min(H) >= 0.0


def test_f1_mu_fixed_point_kkt(rng):
    """MU's fixed points satisfy h_r (HS - M)_r = 0; from a positive start on positive
    data it approaches the NNLS solution."""
    R, I = 3, 30
    S = make_S(rng, R)
    M = rng.random((I, R)) * np.diag(S).mean()
    H = oracle.mu(M, S, np.ones((I, R)), sweeps=20000)
    G = H @ S - M
    assert np.max(np.abs(H * G)) <= 1e-6 * np.max(np.abs(M))
    ref = np.array([nnls_bruteforce(S, M[i]) for i in range(I)])
    assert normwise(H, ref) <= 1e-3


def test_f1_factorize_schemes_on_planted(rng):
    """The planted rank-8 tensor is fitted by all three schemes (HALS/MU slower than ADMM)."""
    p = datagen.planted_tiny(1)
    X = oracle.coalesce(p.dims, p.idx, p.vals)
    start = datagen.perturbed_start(p, 1)
    for upd in (oracle.UPDATE_HALS, oracle.UPDATE_MU):
        r = oracle.factorize(X, start, outer_iters=30, max_iter=1, update=upd)
        assert r["fit"][-1] > 0.99
        assert np.all(np.diff(r["fit"]) > -1e-9)


# --------------------------------------------------------------------- D11 outer stopping rule
def test_D11_fit_tol_stops_at_first_small_change(rng):
    """D11 (L505 "until convergence"): with fit_tol > 0 the outer loop stops after the
    first outer iteration t >= 1 whose fit changed by less than fit_tol.  The stop index
    is read off a fixed-count run of the same problem (the loop is deterministic), and
    the early-stopped run must reproduce that run's prefix bit for bit."""
    dims = (30, 25, 20)
    idx, vals = random_coo(rng, dims, 1500, dup_frac=0.0, neg=False, zeros=False)
    X = oracle.coalesce(dims, idx, vals)
    start = [rng.random((I, 4)) for I in dims]
    T = 8
    full = oracle.factorize(X, start, outer_iters=T, tol=0.0, max_iter=5)
    f = full["fit"]
    assert len(f) == T
    d = np.abs(np.diff(f))                                 # d[t-1] = |fit_t - fit_{t-1}|
    # the first t >= 2 whose change is a new minimum, and a tolerance strictly between
    tstar = next(t for t in range(2, T) if d[t - 1] < np.min(d[:t - 1]))
    tol = np.sqrt(d[tstar - 1] * np.min(d[:tstar - 1]))
    assert d[tstar - 1] < tol < np.min(d[:tstar - 1])
    early = oracle.factorize(X, start, outer_iters=T, tol=0.0, max_iter=5, fit_tol=tol)
    assert len(early["fit"]) == tstar + 1
    assert np.array_equal(early["fit"], f[:tstar + 1])
    ref = oracle.factorize(X, start, outer_iters=tstar + 1, tol=0.0, max_iter=5)
    for a, b in zip(early["factors"], ref["factors"]):
        assert np.array_equal(a, b)
    # a tolerance below every change never stops early; fit_tol = 0 disables the test
    never = oracle.factorize(X, start, outer_iters=T, tol=0.0, max_iter=5, fit_tol=0.5 * np.min(d))
    assert len(never["fit"]) == T


# --------------------------------------------------------------------- D6 normalize_init = 0
def test_D6_unnormalised_start_reaches_the_same_scale_free_update(rng):
    """normalize_init = 0 (the caller's factors used as given, lambda = 1).  The
    converged ADMM update of mode n is the per-row NNLS solution of (M, S) (P2), which
    is scale covariant: with every other factor scaled by a positive diagonal D_k,
    M -> M D and S -> D S D (D = prod D_k), so the NNLS solution is H D^{-1} and its
    column normalisation is unchanged.  One outer iteration with converged updates
    therefore gives the same normalised factors, lambda and fit from raw scaled factors
    (normalize_init = 0) as from the normalised ones (normalize_init = 1).  A dropped or
    misplaced scale anywhere in the branch (Grams, MTTKRP or warm start of raw factors)
    breaks the equality."""
    dims = (14, 11, 9)
    idx, vals = random_coo(rng, dims, 600, dup_frac=0.0, neg=False, zeros=False)
    X = oracle.coalesce(dims, idx, vals)
    R = 3
    base = [oracle.normalize(rng.random((I, R)) + 0.05)[0] for I in dims]
    raw = [b * (0.3 + 4.0 * rng.random(R)) for b in base]           # columns scaled by D_k
    a = oracle.factorize(X, base, outer_iters=1, tol=0.0, max_iter=6000, normalize_init=True)
    b = oracle.factorize(X, raw, outer_iters=1, tol=0.0, max_iter=6000, normalize_init=False)
    for fa, fb in zip(a["factors"], b["factors"]):
        assert normwise(fb, fa) <= 1e-9
    assert normwise(b["lam"][-1], a["lam"][-1]) <= 1e-9
    assert abs(b["fit"][0] - a["fit"][0]) <= 1e-9
    # with few passes the warm start differs (raw vs normalised H), so the branches differ
    a10 = oracle.factorize(X, base, outer_iters=1, tol=0.0, max_iter=3, normalize_init=True)
    b10 = oracle.factorize(X, raw, outer_iters=1, tol=0.0, max_iter=3, normalize_init=False)
    assert normwise(b10["factors"][0], a10["factors"][0]) > 1e-6
    # normalize_init = 0 on already normalised factors is the normalize_init = 1 run on them
    c = oracle.factorize(X, base, outer_iters=2, tol=1e-2, max_iter=10, normalize_init=False)
    d = oracle.factorize(X, [oracle.normalize(f)[0] for f in base], outer_iters=2, tol=1e-2, max_iter=10,
                         normalize_init=True)
    for fc, fd in zip(c["factors"], d["factors"]):
        assert normwise(fc, fd) <= 1e-12


def test_D6_initial_lambda_is_one_in_both_branches(rng):
    """Reading D6: the initial lambda is exactly 1 whether or not the factors are
    normalised first, so the scaled (D4) and literal warm starts coincide for the
    first update of every mode; after one outer iteration the factors (each mode's
    first update, normalised) must be bit-identical across the two warm-start
    readings, and after two (lambda = the previous column norms) they differ."""
    dims = (12, 10, 9)
    idx, vals = random_coo(rng, dims, 500, dup_frac=0.0, neg=False, zeros=False)
    X = oracle.coalesce(dims, idx, vals)
    raw = [rng.random((I, 4)) * 3.0 for I in dims]
    for ni in (False, True):
        w0 = oracle.factorize(X, raw, outer_iters=1, tol=0.0, max_iter=4, normalize_init=ni, warm=oracle.WARM_SCALED)
        w1 = oracle.factorize(X, raw, outer_iters=1, tol=0.0, max_iter=4, normalize_init=ni,
                              warm=oracle.WARM_NORMALIZED)
        for a, b in zip(w0["factors"], w1["factors"]):
            assert np.array_equal(a, b), ni
        v0 = oracle.factorize(X, raw, outer_iters=2, tol=0.0, max_iter=4, normalize_init=ni, warm=oracle.WARM_SCALED)
        v1 = oracle.factorize(X, raw, outer_iters=2, tol=0.0, max_iter=4, normalize_init=ni,
                              warm=oracle.WARM_NORMALIZED)
        assert normwise(v0["factors"][0], v1["factors"][0]) > 1e-6
