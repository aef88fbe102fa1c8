"""Thin ctypes binding of libcstf (include/cstf.h) -- argument marshalling only.

Every numeric step runs in libcstf's sm_100a kernels.  PyTorch supplies device
memory (CUDA tensors), the current stream and process groups.  There is no
fallback: if ``lib/libcstf.so`` is missing this module raises on import.
Function names are the C names.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CSTF_LIB") or os.path.join(_HERE, "lib", "libcstf.so")   # override: experiments
if not os.path.exists(LIB_PATH):
    raise ImportError(f"libcstf.so not built ({LIB_PATH}); run "
                      "`python -m paper_conf_icpp_sohksc24_b200.build` (no CPU fallback exists)")
_lib = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)

c_void_p, c_int, c_int64, c_double = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_double

# status codes
CSTF_OK, CSTF_ERR_INVALID_ARG, CSTF_ERR_UNSUPPORTED, CSTF_ERR_OUT_OF_MEMORY = 0, 1, 2, 3
CSTF_ERR_CUDA, CSTF_ERR_NCCL, CSTF_ERR_NOT_SPD, CSTF_ERR_NUMERIC = 4, 5, 6, 7
CSTF_PROX_NONNEG, CSTF_PROX_IDENTITY, CSTF_PROX_L1, CSTF_PROX_NONNEG_L1, CSTF_PROX_BOX = 0, 1, 2, 3, 4
CSTF_ADMM_AUTO, CSTF_ADMM_STREAMING, CSTF_ADMM_RESIDENT = 0, 1, 2
CSTF_WARM_SCALED, CSTF_WARM_NORMALIZED = 0, 1
CSTF_UPDATE_ADMM, CSTF_UPDATE_HALS, CSTF_UPDATE_MU = 0, 1, 2
PHASES = ("GRAM", "MTTKRP", "UPDATE", "NORMALIZE", "COMM")
NUM_PHASES = len(PHASES)


class CstfError(RuntimeError):
    def __init__(self, status: int, what: str):
        msg = _lib.cstf_last_error_message().decode(errors="replace")
        super().__init__(f"{what}: {_lib.cstf_status_string(status).decode()} -- {msg}")
        self.status = status


class AdmmOpts(ctypes.Structure):
    _fields_ = [("tol", c_double), ("max_iter", c_int), ("rho", c_double), ("prox", c_int),
                ("variant", c_int), ("alpha", c_double)]


class AdmmStats(ctypes.Structure):
    _fields_ = [("iters", c_int), ("rho", c_double), ("r_primal", c_double), ("s_dual", c_double),
                ("normH2", c_double), ("normU2", c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Opts(ctypes.Structure):
    _fields_ = [("R", c_int), ("outer_iters", c_int), ("fit_tol", c_double), ("admm", AdmmOpts),
                ("warm", c_int), ("normalize_init", c_int), ("timing", c_int), ("update", c_int)]


class Report(ctypes.Structure):
    _fields_ = [("outer_done", c_int), ("fit", ctypes.POINTER(c_double)),
                ("admm_iters", ctypes.POINTER(c_int)), ("phase_ms", ctypes.POINTER(c_double)),
                ("mode_phase_ms", ctypes.POINTER(c_double)),
                ("mode_launches", ctypes.POINTER(c_int64))]


def _decl(name, res, args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = args
    return f


_decl("cstf_status_string", ctypes.c_char_p, [c_int])
_decl("cstf_last_error_message", ctypes.c_char_p, [])
_decl("cstf_version", c_int, [])
_decl("cstf_kernel_launch_count", c_int64, [])
_decl("cstf_release_workspace", c_int, [])
_decl("cstf_get_unique_id", c_int, [c_void_p])
_decl("cstf_comm_create", c_int, [c_int, c_int, c_void_p, ctypes.POINTER(c_void_p)])
_decl("cstf_comm_info", c_int, [c_void_p, ctypes.POINTER(c_int), ctypes.POINTER(c_int)])
_ALLREDUCE_FN = ctypes.CFUNCTYPE(c_int, ctypes.POINTER(c_double), c_int64, c_void_p)
_ALLGATHER_FN = ctypes.CFUNCTYPE(c_int, ctypes.POINTER(c_double), ctypes.POINTER(c_double), c_int64, c_void_p)
_decl("cstf_comm_create_host", c_int, [c_int, c_int, _ALLREDUCE_FN, _ALLGATHER_FN, c_void_p, ctypes.POINTER(c_void_p)])
_decl("cstf_comm_loopback", c_int, [c_int, c_void_p])
_decl("cstf_comm_destroy", None, [c_void_p])
_decl("cstf_partition_rows", c_int, [c_int64, c_void_p, c_int, c_void_p, c_void_p])
_decl("cstf_tensor_load_coo", c_int, [c_int, c_void_p, c_int64, c_void_p, c_void_p, c_void_p, c_void_p,
                                      ctypes.POINTER(c_void_p)])
_decl("cstf_tensor_info", c_int, [c_void_p, ctypes.POINTER(c_int), c_void_p, ctypes.POINTER(c_int64),
                                  ctypes.POINTER(c_double), ctypes.POINTER(ctypes.c_uint64)])
_decl("cstf_tensor_export_coo", c_int, [c_void_p, c_void_p, c_void_p])
_decl("cstf_tensor_layout", c_int, [c_void_p, c_int, ctypes.POINTER(c_int64), ctypes.POINTER(c_int64),
                                    ctypes.POINTER(c_int)])
_decl("cstf_tensor_record_bytes", c_int, [c_void_p, c_int, ctypes.POINTER(c_int)])
_decl("cstf_tensor_free", None, [c_void_p])
_decl("cstf_mttkrp", c_int, [c_void_p, c_int, c_int, c_void_p, c_void_p, c_void_p])
_decl("cstf_gram", c_int, [c_void_p, c_int64, c_int, c_void_p, c_void_p, c_void_p])
_decl("cstf_normalize", c_int, [c_void_p, c_int64, c_int, c_void_p, c_void_p, c_void_p, c_void_p])
_decl("cstf_admm_update", c_int, [c_void_p, c_void_p, c_void_p, c_void_p, c_int64, c_int,
                                  ctypes.POINTER(AdmmOpts), c_void_p, ctypes.POINTER(AdmmStats), c_void_p])
_decl("cstf_hals_update", c_int, [c_void_p, c_void_p, c_void_p, c_int64, c_int, c_int, c_void_p])
_decl("cstf_mu_update", c_int, [c_void_p, c_void_p, c_void_p, c_int64, c_int, c_int, c_void_p])
_decl("cstf_factorize", c_int, [c_void_p, ctypes.POINTER(Opts), c_void_p, c_void_p, c_void_p,
                                ctypes.POINTER(Report), c_void_p])
_decl("cstf_factorize_host", c_int, [c_void_p, ctypes.POINTER(Opts), c_void_p, c_void_p, c_void_p,
                                     ctypes.POINTER(Report), c_void_p])

EXPORTED = ["cstf_status_string", "cstf_last_error_message", "cstf_version", "cstf_get_unique_id",
            "cstf_comm_create", "cstf_comm_create_host", "cstf_comm_loopback", "cstf_comm_info", "cstf_comm_destroy",
            "cstf_partition_rows",
            "cstf_tensor_load_coo", "cstf_tensor_info", "cstf_tensor_layout", "cstf_tensor_record_bytes", "cstf_tensor_export_coo", "cstf_tensor_free",
            "cstf_mttkrp", "cstf_gram", "cstf_normalize", "cstf_admm_update", "cstf_hals_update",
            "cstf_mu_update", "cstf_factorize",
            "cstf_factorize_host", "cstf_kernel_launch_count", "cstf_release_workspace"]


def _check(st, what):
    if st != CSTF_OK:
        raise CstfError(st, what)


def _stream(stream=None):
    if stream is not None:
        return c_void_p(stream)
    import torch
    return c_void_p(torch.cuda.current_stream().cuda_stream)


def _dptr(t):
    """Device pointer of a contiguous float64 CUDA tensor (or None)."""
    if t is None:
        return None
    import torch
    assert isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.float64 and t.is_contiguous(), \
        "expected a contiguous float64 CUDA tensor"
    return t.data_ptr()


def _ptr_array(ptrs):
    return (c_void_p * len(ptrs))(*[p if p is not None else None for p in ptrs])


def _comm(comm):
    return comm.handle if comm is not None else None


# ------------------------------------------------------------------- misc
def cstf_version() -> int:
    return _lib.cstf_version()


def cstf_kernel_launch_count() -> int:
    return _lib.cstf_kernel_launch_count()


def cstf_release_workspace() -> None:
    _check(_lib.cstf_release_workspace(), "cstf_release_workspace")


def cstf_partition_rows(counts, nranks: int):
    counts = np.ascontiguousarray(counts, dtype=np.int64)
    I = len(counts)
    owner = np.empty(I, dtype=np.int32)
    local = np.empty(I, dtype=np.int64)
    _check(_lib.cstf_partition_rows(I, counts.ctypes.data, nranks, owner.ctypes.data, local.ctypes.data),
           "cstf_partition_rows")
    return owner, local


class Comm:
    def __init__(self, handle):
        self.handle = handle

    def info(self):
        n, r = c_int(), c_int()
        _check(_lib.cstf_comm_info(self.handle, ctypes.byref(n), ctypes.byref(r)), "cstf_comm_info")
        return n.value, r.value

    def __del__(self, _destroy=_lib.cstf_comm_destroy):
        if getattr(self, "handle", None):
            _destroy(self.handle)
            self.handle = None


def cstf_comm_create_host(group=None) -> Comm:
    """Host-callback communicator over a torch.distributed process group (e.g.
    gloo): lets several processes share one GPU (NCCL needs one GPU per rank).
    The library stages device buffers through host memory; the callbacks only
    move bytes (sum / concatenate) through the process group."""
    import torch
    import torch.distributed as dist
    P = dist.get_world_size(group)
    rank = dist.get_rank(group)

    def allreduce(buf, n, user):
        try:
            t = torch.from_numpy(np.ctypeslib.as_array(buf, shape=(n,)))
            dist.all_reduce(t, group=group)
            return 0
        except Exception:
            return 1

    def allgather(send, recv, n, user):
        try:
            s = torch.from_numpy(np.ctypeslib.as_array(send, shape=(n,)).copy())
            r = torch.from_numpy(np.ctypeslib.as_array(recv, shape=(n * P,)))
            dist.all_gather(list(r.chunk(P)), s, group=group)
            return 0
        except Exception:
            return 1

    cb = (_ALLREDUCE_FN(allreduce), _ALLGATHER_FN(allgather))
    h = c_void_p()
    _check(_lib.cstf_comm_create_host(P, rank, cb[0], cb[1], None, ctypes.byref(h)), "cstf_comm_create_host")
    c = Comm(h.value)
    c._callbacks = cb          # keep the trampolines alive
    return c


def cstf_comm_loopback(nparts: int) -> list:
    """nparts communicators of one process (test backend: one thread per part, one
    GPU); each thread passes its own handle to the library calls."""
    arr = (c_void_p * nparts)()
    _check(_lib.cstf_comm_loopback(int(nparts), arr), "cstf_comm_loopback")
    return [Comm(arr[r]) for r in range(nparts)]


def cstf_comm_create_nccl(group=None) -> Comm:
    """NCCL communicator (one process per GPU); the unique id travels through the
    torch.distributed process group."""
    import torch
    import torch.distributed as dist
    P = dist.get_world_size(group)
    rank = dist.get_rank(group)
    uid = [cstf_get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0, group=group)
    return cstf_comm_create(P, rank, uid[0])


def cstf_get_unique_id() -> bytes:
    buf = (ctypes.c_ubyte * 128)()
    _check(_lib.cstf_get_unique_id(buf), "cstf_get_unique_id")
    return bytes(buf)


def cstf_comm_create(nranks: int, rank: int, uid: bytes) -> Comm:
    buf = (ctypes.c_ubyte * 128).from_buffer_copy(uid)
    h = c_void_p()
    _check(_lib.cstf_comm_create(nranks, rank, buf, ctypes.byref(h)), "cstf_comm_create")
    return Comm(h.value)


# ------------------------------------------------------------------- tensor
class Tensor:
    """Owns a cstf_tensor handle (device-resident mode-sorted store)."""

    def __init__(self, handle):
        self.handle = handle
        info = self.info()
        self.nmodes = info["nmodes"]
        self.dims = info["dims"]

    def info(self):
        n = c_int()
        dims = (c_int64 * 8)()
        nnz = c_int64()
        nx = c_double()
        h = ctypes.c_uint64()
        _check(_lib.cstf_tensor_info(self.handle, ctypes.byref(n), dims, ctypes.byref(nnz), ctypes.byref(nx),
                                     ctypes.byref(h)), "cstf_tensor_info")
        return dict(nmodes=n.value, dims=tuple(dims[:n.value]), nnz=nnz.value, normX2=nx.value, hash=h.value)

    def layout(self, mode: int):
        """(nblk, blk_rows, blk_mode) of the mode copy (nblk = 1: not blocked)."""
        nb, br, bm = c_int64(), c_int64(), c_int()
        _check(_lib.cstf_tensor_layout(self.handle, mode, ctypes.byref(nb), ctypes.byref(br), ctypes.byref(bm)),
               "cstf_tensor_layout")
        return nb.value, br.value, bm.value

    def record_bytes(self, mode: int) -> int:
        """Bytes per nonzero record of the mode copy (16 = packed 4-mode records)."""
        rb = c_int()
        _check(_lib.cstf_tensor_record_bytes(self.handle, mode, ctypes.byref(rb)), "cstf_tensor_record_bytes")
        return rb.value

    def export_coo(self):
        info = self.info()
        nnz = info["nnz"]
        idx = [np.empty(nnz, dtype=np.int32) for _ in range(self.nmodes)]
        vals = np.empty(nnz, dtype=np.float64)
        _check(_lib.cstf_tensor_export_coo(self.handle, _ptr_array([a.ctypes.data for a in idx]),
                                           vals.ctypes.data), "cstf_tensor_export_coo")
        return idx, vals

    def free(self, _free=_lib.cstf_tensor_free):
        # _free bound at definition: at interpreter exit the module global may be gone
        if getattr(self, "handle", None):
            _free(self.handle)
            self.handle = None

    def __del__(self):
        self.free()


def cstf_tensor_load_coo(dims, idx, vals, comm=None, stream=None) -> Tensor:
    N = len(dims)
    dims_a = np.asarray(dims, dtype=np.int64)
    idx = [np.ascontiguousarray(a, dtype=np.int32) for a in idx]
    vals = np.ascontiguousarray(vals, dtype=np.float64)
    h = c_void_p()
    _check(_lib.cstf_tensor_load_coo(N, dims_a.ctypes.data, len(vals), _ptr_array([a.ctypes.data for a in idx]),
                                     vals.ctypes.data, _comm(comm), _stream(stream), ctypes.byref(h)),
           "cstf_tensor_load_coo")
    return Tensor(h.value)


cstf_tensor_info = Tensor.info
cstf_tensor_export_coo = Tensor.export_coo
cstf_tensor_free = Tensor.free


# ------------------------------------------------------------------- kernels
def cstf_mttkrp(X: Tensor, mode: int, factors, M, stream=None):
    R = M.shape[1]
    ptrs = [_dptr(f) if (k != mode and f is not None) else None for k, f in enumerate(factors)]
    _check(_lib.cstf_mttkrp(X.handle, mode, R, _ptr_array(ptrs), _dptr(M), _stream(stream)), "cstf_mttkrp")
    return M


def cstf_gram(H, G, comm=None, stream=None):
    I, R = H.shape
    _check(_lib.cstf_gram(_dptr(H), I, R, _dptr(G), _comm(comm), _stream(stream)), "cstf_gram")
    return G


def cstf_normalize(H, lam, G=None, comm=None, stream=None):
    I, R = H.shape
    _check(_lib.cstf_normalize(_dptr(H), I, R, _dptr(lam), _dptr(G), _comm(comm), _stream(stream)),
           "cstf_normalize")
    return H, lam


def admm_opts(tol=0.0, max_iter=10, rho=0.0, prox=CSTF_PROX_NONNEG, variant=CSTF_ADMM_AUTO,
              alpha=0.0) -> AdmmOpts:
    return AdmmOpts(float(tol), int(max_iter), float(rho), int(prox), int(variant), float(alpha))


def cstf_admm_update(M, S, H, U, tol=0.0, max_iter=10, rho=0.0, prox=CSTF_PROX_NONNEG,
                     variant=CSTF_ADMM_AUTO, comm=None, stream=None, alpha=0.0) -> dict:
    I, R = H.shape
    o = admm_opts(tol, max_iter, rho, prox, variant, alpha)
    st = AdmmStats()
    _check(_lib.cstf_admm_update(_dptr(M), _dptr(S), _dptr(H), _dptr(U), I, R, ctypes.byref(o), _comm(comm),
                                 ctypes.byref(st), _stream(stream)), "cstf_admm_update")
    return st.as_dict()


def make_opts(R, outer_iters=10, fit_tol=0.0, tol=1e-2, max_iter=10, rho=0.0, prox=CSTF_PROX_NONNEG,
              variant=CSTF_ADMM_AUTO, warm=CSTF_WARM_SCALED, normalize_init=True, timing=False,
              alpha=0.0, update=CSTF_UPDATE_ADMM) -> Opts:
    return Opts(int(R), int(outer_iters), float(fit_tol), admm_opts(tol, max_iter, rho, prox, variant, alpha),
                int(warm), int(bool(normalize_init)), int(bool(timing)), int(update))


def cstf_hals_update(M, S, H, sweeps=1, stream=None):
    I, R = H.shape
    _check(_lib.cstf_hals_update(_dptr(M), _dptr(S), _dptr(H), I, R, int(sweeps), _stream(stream)),
           "cstf_hals_update")
    return H


def cstf_mu_update(M, S, H, sweeps=1, stream=None):
    I, R = H.shape
    _check(_lib.cstf_mu_update(_dptr(M), _dptr(S), _dptr(H), I, R, int(sweeps), _stream(stream)),
           "cstf_mu_update")
    return H


class _ReportBufs:
    def __init__(self, outer, N):
        self.fit = np.zeros(outer)
        self.iters = np.zeros(outer * N, dtype=np.int32)
        self.phase = np.zeros(NUM_PHASES)
        self.mode_phase = np.zeros(N * NUM_PHASES)
        self.launches = np.zeros(N * NUM_PHASES, dtype=np.int64)
        self.rep = Report(0, self.fit.ctypes.data_as(ctypes.POINTER(c_double)),
                          self.iters.ctypes.data_as(ctypes.POINTER(c_int)),
                          self.phase.ctypes.data_as(ctypes.POINTER(c_double)),
                          self.mode_phase.ctypes.data_as(ctypes.POINTER(c_double)),
                          self.launches.ctypes.data_as(ctypes.POINTER(c_int64)))

    def result(self, N):
        d = self.rep.outer_done
        return dict(outer_done=d, fit=self.fit[:d].copy(), iters=self.iters.reshape(-1, N)[:d].copy(),
                    phase_ms=dict(zip(PHASES, self.phase.tolist())),
                    mode_phase_ms=self.mode_phase.reshape(N, NUM_PHASES).copy(),
                    mode_launches=self.launches.reshape(N, NUM_PHASES).copy())


def cstf_factorize(X: Tensor, factors, lam, opts: Opts, comm=None, stream=None) -> dict:
    N = X.nmodes
    rb = _ReportBufs(opts.outer_iters, N)
    _check(_lib.cstf_factorize(X.handle, ctypes.byref(opts), _comm(comm), _ptr_array([_dptr(f) for f in factors]),
                               _dptr(lam), ctypes.byref(rb.rep), _stream(stream)), "cstf_factorize")
    return rb.result(N)


def cstf_factorize_host(X: Tensor, host_factors, host_lam, opts: Opts, comm=None, stream=None) -> dict:
    """host_factors: contiguous float64 host arrays (numpy or pinned torch CPU tensors), updated in place."""
    def hp(a):
        if isinstance(a, np.ndarray):
            assert a.dtype == np.float64 and a.flags.c_contiguous
            return a.ctypes.data
        return a.data_ptr()
    N = X.nmodes
    rb = _ReportBufs(opts.outer_iters, N)
    _check(_lib.cstf_factorize_host(X.handle, ctypes.byref(opts), _comm(comm),
                                    _ptr_array([hp(f) for f in host_factors]), hp(host_lam),
                                    ctypes.byref(rb.rep), _stream(stream)), "cstf_factorize_host")
    return rb.result(N)
