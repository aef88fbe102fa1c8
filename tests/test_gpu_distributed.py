"""Partitioned (multi-GPU) path on ONE GPU: P processes share cuda:0 and talk
through the host-callback communicator over gloo (NCCL needs one GPU per rank).
The full distributed code path runs -- row partition, relabelled store, local
MTTKRP and ADMM, all-reduced residual sums and Grams, all-gathered factors --
and rank 0 compares the result with the single-process FP64 oracle."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r'''
import os, sys, json, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import datagen, oracle
from parity_util import compare_iteration_counts
from paper_conf_icpp_sohksc24_b200 import binding as B
dist.init_process_group("gloo")
torch.cuda.set_device(0)
rank, P = dist.get_rank(), dist.get_world_size()
comm = B.cstf_comm_create_nccl() if COMM == "nccl" else B.cstf_comm_create_host()
cfg, scale, R, tol, outer = CASE
c = datagen.CONFIGS[cfg] if scale == 0 else datagen.CONFIGS[cfg].scaled(scale, nnz_factor=scale * 20)
idx, vals = c.generate()
X = B.cstf_tensor_load_coo(c.dims, idx, vals, comm=comm)
start = datagen.init_factors(c.dims, R, c.seed)
F = [torch.from_numpy(f.copy()).cuda() for f in start]
lam = torch.zeros(R, dtype=torch.float64, device="cuda")
rep = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=outer, tol=tol, max_iter=10, timing=True), comm=comm)
rep2 = B.cstf_factorize(X, [torch.from_numpy(f.copy()).cuda() for f in start], lam.clone(),
                        B.make_opts(R, outer_iters=outer, tol=tol, max_iter=10), comm=comm)   # back-to-back calls
torch.cuda.synchronize()
assert np.array_equal(rep["fit"], rep2["fit"]), (rep["fit"], rep2["fit"])
out = {"fit": rep["fit"].tolist(), "iters": rep["iters"].tolist(), "comm_ms": rep["phase_ms"]["COMM"],
       "nblk": [X.layout(n)[0] for n in range(len(c.dims))]}
if rank == 0:
    oracle.set_threads(len(os.sched_getaffinity(0)))    # torchrun runs every rank with OMP_NUM_THREADS=1
    ref = oracle.coalesce(c.dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=outer, tol=tol, max_iter=10)
    ncmp, tie = compare_iteration_counts(rep["iters"], orc, tol if tol > 0 else 1e-2)
    out["ncmp"] = ncmp; out["tie"] = tie is not None
    out["fit_rel"] = float(np.max(np.abs(rep["fit"] - orc["fit"]) / np.abs(orc["fit"])))
    out["fac_rel"] = max(float(np.max(np.abs(f.cpu().numpy() - g)) / np.max(np.abs(g)))
                         for f, g in zip(F, orc["factors"]))
    out["lam_rel"] = float(np.max(np.abs(lam.cpu().numpy() - orc["lam"][-1])) / np.max(np.abs(orc["lam"][-1])))
sys.stdout.write(f"RESULT {rank} " + json.dumps(out) + "\n"); sys.stdout.flush()   # one write: ranks share the pipe
dist.destroy_process_group()
'''


def run(tmp_path, nproc, case, port, comm="host"):
    p = tmp_path / "dist_case.py"
    p.write_text(f"ROOT = {ROOT!r}\nCASE = {case!r}\nCOMM = {comm!r}\n" + SCRIPT)
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", PYTHONPATH=ROOT)
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
                        "--master-addr=127.0.0.1", f"--master-port={port}", str(p)],
                       env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-5000:]
    import json
    res = {}
    for line in r.stdout.splitlines():
        if line.startswith("RESULT"):
            _, rk, js = line.split(" ", 2)
            res[int(rk)] = json.loads(js)
    assert len(res) == nproc
    return res


@pytest.mark.parametrize("nproc,case,port,peer", [
    (2, ("nell2", 40, 16, 1e-2, 5), 29611, "1"),
    (3, ("enron", 60, 8, 1e-2, 5), 29612, "1"),
    (2, ("delicious", 2000, 32, 0.0, 3), 29613, "1"),     # eps = 0: ADMM epilogue peer stores (f4)
    (3, ("nell2", 40, 32, 0.0, 4), 29614, "1"),
    (3, ("nell2", 40, 32, 0.0, 4), 29615, "0"),           # same case through the plain all-gather
    (1, ("nell2", 40, 32, 0.0, 4), 29616, "nccl"),        # a real NCCL communicator of one rank
    (1, ("enron", 60, 8, 1e-2, 5), 29617, "nccl"),
    (2, ("nell2", 40, 32, 0.0, 4), 29618, "blk"),          # L2-blocked partitioned copies (forced)
    (3, ("enron", 60, 16, 1e-2, 5), 29619, "blk"),
    (2, ("delicious", 1000, 32, 0.0, 3), 29620, "hot"),   # hot-row tables over internal labels (forced)
    (3, ("delicious", 1000, 16, 1e-2, 4), 29622, "hot"),
    # full size (scale 0), the bench protocol (eps = 0, 10 passes, one outer iteration):
    # configs[2] Enron-shaped (54M nonzeros) and configs[3] Delicious-shaped (140M) on 2 ranks
    (2, ("enron", 0, 32, 0.0, 1), 29623, "1"),
    (2, ("delicious", 0, 32, 0.0, 1), 29624, "1"),
])
def test_partitioned_factorize_matches_oracle(tmp_path, nproc, case, port, peer, monkeypatch):
    """peer: CSTF_PEER_STORE for the host communicator, or "nccl" (one rank: the
    NCCL transport -- dlopen, unique id, init, all-reduce, all-gather -- and the
    partitioned layout with P = 1, the only NCCL job one GPU can run)."""
    comm = "nccl" if peer == "nccl" else "host"
    monkeypatch.setenv("CSTF_PEER_STORE", "1" if peer in ("nccl", "blk", "hot") else peer)
    if peer == "blk":
        monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "64")
    if peer == "hot":
        monkeypatch.setenv("CSTF_HOT_ROWS", "150")
    res = run(tmp_path, nproc, case, port, comm)
    r0 = res[0]
    for rk in range(1, nproc):          # every rank took the same decisions
        assert res[rk]["fit"] == r0["fit"] and res[rk]["iters"] == r0["iters"]
    assert r0["fit_rel"] <= 1e-6
    if peer == "blk":
        assert all(max(res[rk]["nblk"]) > 1 for rk in range(nproc))     # some mode copy L2-blocked
    if nproc > 1 and peer in ("1", "blk", "hot") and case[3] == 0.0 and case[2] <= 32:
        assert r0["comm_ms"] == 0.0          # no separate all-gather ran: rows were peer-stored
    if not r0["tie"]:
        assert r0["fac_rel"] <= 1e-6 and r0["lam_rel"] <= 1e-6


# ----------------------------------------------------------------- loopback (threads)
def _loopback_run(B, torch, nparts, c, R, tol, outer, fail_rank=None):
    """nparts threads of this process, one cstf_comm_loopback handle and one stream each."""
    import threading
    import datagen
    idx, vals = c.generate()
    start = datagen.init_factors(c.dims, R, c.seed)
    comms = B.cstf_comm_loopback(nparts)
    out = [None] * nparts

    def part(r):
        torch.cuda.set_device(0)
        s = torch.cuda.Stream()
        try:
            with torch.cuda.stream(s):
                X = B.cstf_tensor_load_coo(c.dims, idx, vals, comm=comms[r])
                F = [torch.from_numpy(f.copy()).cuda() for f in start]
                lam = torch.zeros(R, dtype=torch.float64, device="cuda")
                rep = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=outer, tol=tol, max_iter=10),
                                       comm=comms[r])
                s.synchronize()
                out[r] = ("ok", rep, [f.cpu().numpy() for f in F], lam.cpu().numpy())
        except B.CstfError as e:
            out[r] = ("err", e.status, str(e))

    th = [threading.Thread(target=part, args=(r,)) for r in range(nparts)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not any(t.is_alive() for t in th), "a loopback part hung"
    return out, idx, vals, start


@pytest.mark.parametrize("nparts,cfg,scale,R,tol", [(2, "nell2", 40, 16, 1e-2), (3, "enron", 60, 32, 0.0)])
def test_loopback_threads_match_oracle(nparts, cfg, scale, R, tol):
    """cstf_comm_loopback: nparts threads of one process run the partitioned algorithm
    on one GPU (same-process CUDA IPC is refused, so the agreed fallback all-gather
    runs); every part matches the single-process oracle and takes the same decisions."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import numpy as np
    import datagen
    import oracle
    from parity_util import compare_iteration_counts
    from paper_conf_icpp_sohksc24_b200 import binding as B
    c = datagen.CONFIGS[cfg] if scale == 0 else datagen.CONFIGS[cfg].scaled(scale, nnz_factor=scale * 20)
    out, idx, vals, start = _loopback_run(B, torch, nparts, c, R, tol, 4)
    assert all(o[0] == "ok" for o in out), out
    ref = oracle.coalesce(c.dims, idx, vals)
    orc = oracle.factorize(ref, start, outer_iters=4, tol=tol, max_iter=10)
    for o in out:
        assert np.array_equal(o[1]["fit"], out[0][1]["fit"]) and np.array_equal(o[1]["iters"], out[0][1]["iters"])
    n, tie = compare_iteration_counts(out[0][1]["iters"], orc, tol if tol > 0 else 1e-2)
    assert tie is None
    assert np.max(np.abs(out[0][1]["fit"] - orc["fit"]) / np.abs(orc["fit"])) <= 1e-6
    for a, b in zip(out[0][2], orc["factors"]):
        assert np.max(np.abs(a - b)) / np.max(np.abs(b)) <= 1e-6


def test_loopback_injected_failure_same_status_on_every_part(monkeypatch):
    """SURVEY s8(b) error semantics: part 1 fails its setup (CSTF_TEST_FAIL_RANK=1,
    simulated out-of-memory); every part returns CSTF_ERR_OUT_OF_MEMORY, nobody
    hangs, and the same handles then run a clean factorisation."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import datagen
    from paper_conf_icpp_sohksc24_b200 import binding as B
    c = datagen.CONFIGS["nell2"].scaled(80, nnz_factor=4000)
    monkeypatch.setenv("CSTF_TEST_FAIL_RANK", "1")
    out, *_ = _loopback_run(B, torch, 3, c, 8, 1e-2, 2)
    assert [o[0] for o in out] == ["err"] * 3, out
    assert all(o[1] == B.CSTF_ERR_OUT_OF_MEMORY for o in out), out
    assert "another rank failed" in out[0][2] and "injected" in out[1][2]
    monkeypatch.delenv("CSTF_TEST_FAIL_RANK")
    out, *_ = _loopback_run(B, torch, 3, c, 8, 1e-2, 2)
    assert all(o[0] == "ok" for o in out), out


REALLOC = r'''
import os, sys, json, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import datagen, oracle
from paper_conf_icpp_sohksc24_b200 import binding as B
dist.init_process_group("gloo")
torch.cuda.set_device(0)
rank, P = dist.get_rank(), dist.get_world_size()
comm = B.cstf_comm_create_host()
if rank == 0:
    oracle.set_threads(len(os.sched_getaffinity(0)))    # torchrun runs every rank with OMP_NUM_THREADS=1
res = []
# small -> larger (replica buffer re-allocated, peer mappings refreshed) -> small again
for cfg, scale, R in (("nell2", 80, 16), ("enron", 30, 32), ("nell2", 80, 16), ("nell2", 40, 32)):
    c = datagen.CONFIGS[cfg] if scale == 0 else datagen.CONFIGS[cfg].scaled(scale, nnz_factor=scale * 20)
    idx, vals = c.generate()
    X = B.cstf_tensor_load_coo(c.dims, idx, vals, comm=comm)
    start = datagen.init_factors(c.dims, R, 3)
    F = [torch.from_numpy(f.copy()).cuda() for f in start]
    lam = torch.zeros(R, dtype=torch.float64, device="cuda")
    rep = B.cstf_factorize(X, F, lam, B.make_opts(R, outer_iters=3, tol=0.0, max_iter=10, timing=True), comm=comm)
    torch.cuda.synchronize()
    r = {"fit": rep["fit"].tolist(), "comm_ms": rep["phase_ms"]["COMM"]}
    if rank == 0:
        orc = oracle.factorize(oracle.coalesce(c.dims, idx, vals), start, outer_iters=3, tol=0.0, max_iter=10)
        r["fit_rel"] = float(np.max(np.abs(rep["fit"] - orc["fit"]) / np.abs(orc["fit"])))
        r["fac_rel"] = max(float(np.max(np.abs(f.cpu().numpy() - g)) / np.max(np.abs(g)))
                           for f, g in zip(F, orc["factors"]))
    res.append(r)
sys.stdout.write(f"RESULT {rank} " + json.dumps(res) + "\n"); sys.stdout.flush()
dist.destroy_process_group()
'''


def test_peer_stores_across_reallocations(tmp_path, monkeypatch):
    """Back-to-back factorisations of tensors of different sizes on 2 processes with
    peer stores (f4): the replica buffer is re-allocated, every call re-decides the IPC
    mapping collectively, and every call matches the oracle without a separate
    all-gather (ADVICE r01 api.cu:75)."""
    monkeypatch.setenv("CSTF_PEER_STORE", "1")
    p = tmp_path / "realloc.py"
    p.write_text(f"ROOT = {ROOT!r}\n" + REALLOC)
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", PYTHONPATH=ROOT)
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr=127.0.0.1", "--master-port=29621", str(p)],
                       env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-5000:]
    import json
    res = {}
    for line in r.stdout.splitlines():
        if line.startswith("RESULT"):
            _, rk, js = line.split(" ", 2)
            res[int(rk)] = json.loads(js)
    assert len(res) == 2
    for a, b in zip(res[0], res[1]):
        assert a["fit"] == b["fit"]
    for a in res[0]:
        assert a["fit_rel"] <= 1e-6 and a["fac_rel"] <= 1e-6
        assert a["comm_ms"] == 0.0          # rows went to the replicas by peer stores
