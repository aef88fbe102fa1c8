"""Packed 16-byte records of 4-mode mode copies (store.cu
decide_pack, mttkrp.cu pk_field): {uint64 bit-packed indices of the three gathered
modes (plus hot-row flags), f64 value} instead of {3 x int32, pad, f64}.

  * chosen where the three fields fit 64 bits (an L2-blocked copy stores its blocked
    slot relative to the block) and the copy has >= 16 nonzeros per (virtual) row
    (CSTF_PACK=2 forces it wherever the fields fit);
  * MTTKRP on packed copies equals the 32-byte-record copies bit for bit (same nonzero
    order, same kernels and arithmetic) for the fast kernel (R = 16 / 32 / 64, with and
    without hot-row slots, both group widths) and the generic kernel (R = 5), and the
    FP64 oracle (Fig. 2) within 1e-9 normwise;
  * export of a packed store with hot-row slots returns the canonical tensor;
  * a factorisation on packed copies equals the unpacked one bit for bit.
"""
import numpy as np
import pytest

import datagen
import oracle

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
    den = np.max(np.abs(b))
    return float(np.max(np.abs(a - b)) / (den if den > 0 else 1.0))


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def bits(n):
    return max(1, int(n - 1).bit_length())


@pytest.fixture(scope="module")
def delicious_small():
    """Delicious-shaped (gammas 2/2/3/1) / 100 per mode, 1.4M nonzeros."""
    c = datagen.CONFIGS["delicious"].scaled(100, nnz_factor=100)
    idx, vals = c.generate()
    return c, idx, vals, oracle.coalesce(c.dims, idx, vals)


def mttkrp_all(B, X, dims, Fd, R):
    outs = []
    for n in range(len(dims)):
        M = cu(np.full((dims[n], R), np.nan))
        B.cstf_mttkrp(X, n, Fd, M)
        outs.append(host(M).copy())
    return outs


@pytest.mark.parametrize("hot", [None, "300"])
@pytest.mark.parametrize("R,g", [(32, None), (32, "0"), (16, None), (64, None), (5, None)])
def test_packed_mttkrp_bitwise_and_oracle(B, delicious_small, hot, R, g, monkeypatch):
    c, idx, vals, ref = delicious_small
    monkeypatch.setenv("CSTF_PACK", "2")
    if hot:
        monkeypatch.setenv("CSTF_HOT_ROWS", hot)
    if g is not None:
        monkeypatch.setenv("CSTF_MTTKRP_G", g)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    monkeypatch.setenv("CSTF_PACK", "0")
    Xu = B.cstf_tensor_load_coo(c.dims, idx, vals)
    for n in range(4):
        assert X.record_bytes(n) == 16 and Xu.record_bytes(n) == 32, n
    F = datagen.init_factors(c.dims, R, 21)
    Fd = [cu(f) for f in F]
    a = mttkrp_all(B, X, c.dims, Fd, R)
    b = mttkrp_all(B, Xu, c.dims, Fd, R)
    for n in range(4):
        assert np.array_equal(a[n], b[n]), n
        assert normwise(a[n], oracle.mttkrp(ref, n, F)) <= TOL, n


def test_packed_only_where_fields_fit(B, monkeypatch):
    """Mode 0 of a tensor whose three other modes need 22 bits each (66 > 64) keeps the
    32-byte records; the other modes (one 2-bit field) pack (forced past the row-length
    rule; L2 blocks off, which would make mode 0's longest slot block-relative and fit).
    MTTKRP of both kinds against the oracle."""
    monkeypatch.setenv("CSTF_PACK", "2")
    monkeypatch.setenv("CSTF_L2_BLOCK", "0")
    dims = (3, 3_000_000, 2_500_000, 2_200_000)
    need = [sum(bits(dims[k]) for k in range(4) if k != n) for n in range(4)]
    assert need[0] > 64 and all(x <= 64 for x in need[1:])
    idx, vals = datagen.coo(dims, (1, 2, 2, 3), 200_000, 41)
    X = B.cstf_tensor_load_coo(dims, idx, vals)
    assert [X.record_bytes(n) for n in range(4)] == [32, 16, 16, 16]
    ref = oracle.coalesce(dims, idx, vals)
    R = 8
    F = datagen.init_factors(dims, R, 42)
    Fd = [cu(f) for f in F]
    for n, got in enumerate(mttkrp_all(B, X, dims, Fd, R)):
        assert normwise(got, oracle.mttkrp(ref, n, F)) <= TOL, n


@pytest.mark.parametrize("hot", [None, "300"])
@pytest.mark.parametrize("R", [32, 64, 5])
def test_l2_blocked_copies_pack_block_relative(B, delicious_small, hot, R, monkeypatch):
    """L2-blocked copies (forced 20,000-row blocks) pack too, their blocked slot stored as
    the row within its block (the kernel adds the block's first row of the current virtual
    row): MTTKRP bit for bit equal to the 32-byte copies and to the oracle within 1e-9,
    export (mode 0 is blocked here) back to the canonical tensor."""
    c, idx, vals, ref = delicious_small
    monkeypatch.setenv("CSTF_PACK", "2")
    monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "20000")
    if hot:
        monkeypatch.setenv("CSTF_HOT_ROWS", hot)
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    monkeypatch.setenv("CSTF_PACK", "0")
    Xu = B.cstf_tensor_load_coo(c.dims, idx, vals)
    blocked = [X.layout(n)[0] > 1 for n in range(4)]
    assert blocked[0] and sum(blocked) >= 2
    assert [X.record_bytes(n) for n in range(4)] == [16] * 4
    assert [Xu.record_bytes(n) for n in range(4)] == [32] * 4
    F = datagen.init_factors(c.dims, R, 23)
    Fd = [cu(f) for f in F]
    a = mttkrp_all(B, X, c.dims, Fd, R)
    b = mttkrp_all(B, Xu, c.dims, Fd, R)
    for n in range(4):
        assert np.array_equal(a[n], b[n]), n
        assert normwise(a[n], oracle.mttkrp(ref, n, F)) <= TOL, n
    gi, gv = X.export_coo()
    for m in range(4):
        assert np.array_equal(gi[m], ref.idx[m]), m
    assert np.array_equal(gv, ref.vals)


def test_packed_export_with_hot_rows(B, delicious_small, monkeypatch):
    """Export decodes packed records, hot-row slots included, to the canonical tensor."""
    c, idx, vals, ref = delicious_small
    monkeypatch.setenv("CSTF_HOT_ROWS", "300")
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    assert X.record_bytes(0) == 16      # mode 0: 263 nonzeros per row, packed by default
    gi, gv = X.export_coo()
    for m in range(4):
        assert np.array_equal(gi[m], ref.idx[m]), m
    assert np.array_equal(gv, ref.vals)
    assert X.info()["hash"] == ref.hash


def test_packed_factorize_bitwise(B, delicious_small, monkeypatch):
    """Two outer iterations (R = 32, eps = 0, 10 passes, hot-row slots forced) on packed
    and on 32-byte copies: identical factors, lambda and fits; fit against the oracle."""
    c, idx, vals, ref = delicious_small
    monkeypatch.setenv("CSTF_HOT_ROWS", "300")
    R = 32
    start = datagen.init_factors(c.dims, R, c.seed)
    res = []
    for pack in ("2", "0"):
        monkeypatch.setenv("CSTF_PACK", pack)
        X = B.cstf_tensor_load_coo(c.dims, idx, vals)
        assert X.record_bytes(0) == (16 if pack == "2" else 32)
        F = [cu(f) for f in start]
        lam = cu(np.zeros(R))
        out = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=2, tol=0.0, max_iter=10))
        res.append(([host(f).copy() for f in F], host(lam).copy(), np.array(out["fit"])))
    for a, b in zip(res[0][0], res[1][0]):
        assert np.array_equal(a, b)
    assert np.array_equal(res[0][1], res[1][1]) and np.array_equal(res[0][2], res[1][2])
    orc = oracle.factorize(ref, start, outer_iters=2, tol=0.0, max_iter=10)
    assert np.max(np.abs(res[0][2] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6


def test_default_rule_skips_short_rows(B, delicious_small):
    """Default rule: copies with < 16 nonzeros per row keep 32-byte records (Delicious-
    shaped mode 1, ~8 per row), longer-row copies pack."""
    c, idx, vals, ref = delicious_small
    X = B.cstf_tensor_load_coo(c.dims, idx, vals)
    for n in range(4):
        want = 16 if ref.vals.size >= 16 * c.dims[n] else 32
        assert X.record_bytes(n) == want, n
