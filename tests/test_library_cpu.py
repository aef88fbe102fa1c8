"""Host-side checks of libcstf (no GPU): the library builds for sm_100a, loads,
exports every symbol include/cstf.h declares, validates arguments before
touching the device, and its row partitioner (multi-GPU host logic) is a
deterministic, balanced, complete partition -- also across a 2-rank gloo world."""
import ctypes
import os
import re
import subprocess
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_sohksc24_b200 import build
    build.build()
    from paper_conf_icpp_sohksc24_b200 import binding
    return binding


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "cstf.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(cstf_[a-z_0-9]+)\s*\(", txt)))


def test_header_symbols_exported(lib):
    syms = header_symbols()
    assert len(syms) >= 18
    so = ctypes.CDLL(lib.LIB_PATH)
    for s in syms:
        assert hasattr(so, s), f"{s} declared in include/cstf.h but not exported"
    assert set(lib.EXPORTED) <= set(syms)


def test_sm100a_cubin(lib):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", lib.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "DMMA" in sass          # FP64 tensor-core product in the ADMM kernel


def test_status_strings_and_version(lib):
    assert lib._lib.cstf_status_string(6) == b"CSTF_ERR_NOT_SPD"
    assert lib.cstf_version() == 1


def test_argument_validation_without_gpu(lib):
    h = ctypes.c_void_p()
    dims = (ctypes.c_int64 * 1)(5)
    st = lib._lib.cstf_tensor_load_coo(1, dims, 0, None, None, None, None, ctypes.byref(h))
    assert st == lib.CSTF_ERR_INVALID_ARG
    assert b"nmodes" in lib._lib.cstf_last_error_message()
    dims3 = (ctypes.c_int64 * 3)(5, 0, 3)
    st = lib._lib.cstf_tensor_load_coo(3, dims3, 0, None, None, None, None, ctypes.byref(h))
    assert st == lib.CSTF_ERR_INVALID_ARG
    st = lib._lib.cstf_tensor_load_coo(3, dims3, 1 << 33, None, None, None, None, ctypes.byref(h))
    assert st == lib.CSTF_ERR_UNSUPPORTED
    o = lib.admm_opts(max_iter=0)
    st = lib._lib.cstf_admm_update(None, ctypes.c_void_p(8), None, None, 0, 8, ctypes.byref(o), None, None, None)
    assert st == lib.CSTF_ERR_INVALID_ARG
    st = lib._lib.cstf_gram(ctypes.c_void_p(8), 4, 129, ctypes.c_void_p(8), None, None)
    assert st == lib.CSTF_ERR_UNSUPPORTED
    # the box prox needs a positive upper bound (reading D25); checked before any device work
    d = ctypes.c_void_p(8)
    o = lib.admm_opts(max_iter=10, prox=lib.CSTF_PROX_BOX, alpha=0.0)
    st = lib._lib.cstf_admm_update(d, d, d, d, 16, 8, ctypes.byref(o), None, None, None)
    assert st == lib.CSTF_ERR_INVALID_ARG and b"box" in lib._lib.cstf_last_error_message()
    o = lib.admm_opts(max_iter=10, prox=5)
    assert lib._lib.cstf_admm_update(d, d, d, d, 16, 8, ctypes.byref(o), None, None, None) == lib.CSTF_ERR_INVALID_ARG
    rb = ctypes.c_int()
    assert lib._lib.cstf_tensor_record_bytes(None, 0, ctypes.byref(rb)) == lib.CSTF_ERR_INVALID_ARG


def check_partition(counts, P, owner, local):
    I = len(counts)
    rows_per = np.bincount(owner, minlength=P)
    assert rows_per.max() - rows_per.min() <= 1                       # equal row counts
    for r in range(P):
        loc = np.sort(local[owner == r])
        assert np.array_equal(loc, np.arange(len(loc)))               # dense local ids
    nnz_per = np.bincount(owner, weights=counts, minlength=P)
    assert nnz_per.max() - nnz_per.min() <= counts.max()              # snake deal bound


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_partition_rows(lib, P):
    rng = np.random.default_rng(P)
    counts = (rng.pareto(1.2, 1001) * 10).astype(np.int64)
    owner, local = lib.cstf_partition_rows(counts, P)
    check_partition(counts, P, owner, local)
    o2, l2 = lib.cstf_partition_rows(counts, P)
    assert np.array_equal(owner, o2) and np.array_equal(local, l2)


def test_partition_rows_gloo_world2(tmp_path):
    """Two processes (gloo) each compute their share; the shares are disjoint,
    cover every row and agree on the global map (all_gather)."""
    script = tmp_path / "w.py"
    script.write_text(f"""
import os, sys, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, {ROOT!r})
from paper_conf_icpp_sohksc24_b200 import binding
dist.init_process_group("gloo")
r, P = dist.get_rank(), dist.get_world_size()
import datagen
idx, v = datagen.coo((3000, 700, 1100), (2, 3, 1), 50000, 11)
ok = True
for n, I in enumerate((3000, 700, 1100)):
    counts = np.bincount(idx[n], minlength=I).astype(np.int64)
    owner, local = binding.cstf_partition_rows(counts, P)
    mine = torch.tensor(np.flatnonzero(owner == r))
    sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(P)]
    dist.all_gather(sizes, torch.tensor([len(mine)]))
    m = max(int(s) for s in sizes)
    pad = torch.full((m,), -1, dtype=torch.int64); pad[:len(mine)] = mine
    parts = [torch.empty(m, dtype=torch.int64) for _ in range(P)]
    dist.all_gather(parts, pad)
    allrows = torch.cat([p[p >= 0] for p in parts]).numpy()
    ok &= len(allrows) == I and len(np.unique(allrows)) == I
    ok &= max(int(s) for s in sizes) - min(int(s) for s in sizes) <= 1
    nnz_mine = torch.tensor([float(counts[owner == r].sum())])
    dist.all_reduce(nnz_mine)
    ok &= int(nnz_mine.item()) == 50000
print("OK" if ok else "BAD", flush=True)
dist.destroy_process_group()
""")
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                          "--master-addr=127.0.0.1", "--master-port=29533", str(script)],
                         env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-3000:]
    assert out.stdout.count("OK") == 2, out.stdout + out.stderr[-2000:]


def test_loopback_comms_without_gpu(lib):
    """cstf_comm_loopback (SURVEY s8(b) test backend): nparts handles with ranks
    0..nparts-1 of one group, created and destroyed without a device."""
    comms = lib.cstf_comm_loopback(3)
    assert [c.info() for c in comms] == [(3, 0), (3, 1), (3, 2)]
    del comms
    arr = (ctypes.c_void_p * 1)()
    assert lib._lib.cstf_comm_loopback(0, arr) == lib.CSTF_ERR_INVALID_ARG
    assert lib._lib.cstf_comm_loopback(65, arr) == lib.CSTF_ERR_INVALID_ARG


def test_ablation_library_exports():
    """The bench-only Fig. 4 library (include/cstf_ablation.h) builds and exports its ABI."""
    from paper_conf_icpp_sohksc24_b200 import build
    path = build.build_ablation()
    so = ctypes.CDLL(path)
    txt = re.sub(r"/\*.*?\*/", "", open(os.path.join(ROOT, "include", "cstf_ablation.h")).read(), flags=re.S)
    syms = set(re.findall(r"\b(cstf_[a-z_0-9]+)\s*\(", txt))
    assert syms == {"cstf_ablation_admm", "cstf_ablation_last_error", "cstf_ablation_last_calls",
                    "cstf_ablation_fp64_peak"}
    for s in syms:
        assert hasattr(so, s)
    so.cstf_ablation_admm.restype = ctypes.c_int
    so.cstf_ablation_last_error.restype = ctypes.c_char_p
    rc = so.cstf_ablation_admm(7, None, None, None, None, ctypes.c_int64(10), 8, 10, None, None)
    assert rc != 0 and b"arm" in so.cstf_ablation_last_error()
