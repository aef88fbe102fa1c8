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
c = datagen.CONFIGS[cfg].scaled(scale, nnz_factor=scale * 20)
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
])
def test_partitioned_factorize_matches_oracle(tmp_path, nproc, case, port, peer, monkeypatch):
    """peer: CSTF_PEER_STORE for the host communicator, or "nccl" (one rank: the
    NCCL transport -- dlopen, unique id, init, all-reduce, all-gather -- and the
    partitioned layout with P = 1, the only NCCL job one GPU can run)."""
    comm = "nccl" if peer == "nccl" else "host"
    monkeypatch.setenv("CSTF_PEER_STORE", "1" if peer in ("nccl", "blk") else peer)
    if peer == "blk":
        monkeypatch.setenv("CSTF_L2_BLOCK_ROWS", "64")
    res = run(tmp_path, nproc, case, port, comm)
    r0 = res[0]
    for rk in range(1, nproc):          # every rank took the same decisions
        assert res[rk]["fit"] == r0["fit"] and res[rk]["iters"] == r0["iters"]
    assert r0["fit_rel"] <= 1e-6
    if peer == "blk":
        assert all(max(res[rk]["nblk"]) > 1 for rk in range(nproc))     # some mode copy L2-blocked
    if nproc > 1 and peer in ("1", "blk") and case[3] == 0.0 and case[2] <= 32:
        assert r0["comm_ms"] == 0.0          # no separate all-gather ran: rows were peer-stored
    if not r0["tie"]:
        assert r0["fac_rel"] <= 1e-6 and r0["lam_rel"] <= 1e-6
