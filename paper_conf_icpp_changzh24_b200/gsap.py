"""Thin ctypes binding of libgsap.so (include/gsap.h): argument marshalling only.

Every step of the hot path runs in the CUDA kernels of libgsap.so.  There is no
CPU fallback: importing works without a GPU (for the ABI checks), but every
call needs the built library and an sm_100 device, and raises otherwise.

Arrays may be numpy arrays (host) or torch tensors (host or CUDA); outputs are
allocated as numpy arrays unless ``device=True`` (torch CUDA tensors).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GSAP_LIB", os.path.join(HERE, "libgsap.so"))

GSAP_OK, GSAP_EINVAL, GSAP_ENOMEM, GSAP_ECUDA, GSAP_ENCCL, GSAP_ESTATE, GSAP_EUNSUPPORTED = range(7)
GSAP_MERGE, GSAP_MOVE = 0, 1
TRACE_COLS = 12                 # GSAP_TRACE_COLS (gsap.h)
STATUS_NAMES = ["GSAP_OK", "GSAP_EINVAL", "GSAP_ENOMEM", "GSAP_ECUDA", "GSAP_ENCCL", "GSAP_ESTATE",
                "GSAP_EUNSUPPORTED"]

EXPORTED = ["gsap_default_params", "gsap_last_error", "gsap_partition", "gsap_create", "gsap_destroy",
            "gsap_set_partition", "gsap_get_partition", "gsap_update_blockmodel", "gsap_propose",
            "gsap_delta_mdl", "gsap_select_merges", "gsap_apply_moves", "gsap_move_batch",
            "gsap_merge_phase", "gsap_mcmc_phase", "gsap_mdl", "gsap_get_blockmodel", "gsap_get_stats", "gsap_reset_stats",
            "gsap_sync", "gsap_run", "gsap_nccl_unique_id", "gsap_shard_slice", "gsap_shard_plan"]


class gsap_params(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("beta", C.c_double), ("reduction_rate", C.c_double),
                ("num_proposals", C.c_int32), ("max_nodal_itr", C.c_int32), ("thresh1", C.c_double),
                ("thresh2", C.c_double), ("window", C.c_int32), ("num_batches", C.c_int32),
                ("model_term", C.c_int32), ("max_rounds", C.c_int32), ("profile", C.c_int32),
                ("cuda_graphs", C.c_int32), ("dense_max_B", C.c_int32), ("sparse_coop", C.c_int32), ("dense_coop", C.c_int32),
                ("sel_small", C.c_int32), ("move_sorted", C.c_int32), ("sim_ranks", C.c_int32),
                ("incremental", C.c_int32), ("proposal_mode", C.c_int32),
                ("line_sort", C.c_int32)]


class gsap_dist(C.Structure):
    _fields_ = [("nranks", C.c_int32), ("rank", C.c_int32), ("device", C.c_int32),
                ("nccl_id", C.c_uint8 * 128)]


class gsap_stats(C.Structure):
    _fields_ = [("t_total", C.c_double), ("t_setup", C.c_double), ("t_merge", C.c_double),
                ("t_move", C.c_double), ("t_mdl", C.c_double),
                ("n_move_prop", C.c_int64), ("n_move_acc", C.c_int64), ("n_merge_prop", C.c_int64),
                ("rounds", C.c_int32), ("mcmc_itr_total", C.c_int32), ("B_final", C.c_int32),
                ("gpu_launches", C.c_int64),
                ("k_move_ms", C.c_double), ("k_move_bytes", C.c_double), ("k_move_launches", C.c_int64),
                ("k_rebuild_ms", C.c_double), ("k_rebuild_bytes", C.c_double),
                ("k_rebuild_launches", C.c_int64),
                ("k_merge_ms", C.c_double), ("k_merge_bytes", C.c_double), ("k_merge_launches", C.c_int64),
                ("k_mdl_ms", C.c_double), ("k_mdl_launches", C.c_int64),
                ("t_rebuild", C.c_double), ("t_comm", C.c_double), ("n_move_eval", C.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class GsapError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


_lib = None


def lib():
    """Load libgsap.so; raise if it was not built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libgsap.so not built ({LIB_PATH}); run __graft_entry__.build()")
        L = C.CDLL(LIB_PATH)
        vp, i32, u32, i64p = C.c_void_p, C.c_int32, C.c_uint32, C.POINTER(C.c_int64)
        L.gsap_default_params.argtypes = [C.POINTER(gsap_params)]
        L.gsap_default_params.restype = None
        L.gsap_last_error.restype = C.c_char_p
        L.gsap_partition.argtypes = [i32, vp, vp, vp, C.POINTER(gsap_params), C.POINTER(gsap_dist), vp,
                                     C.POINTER(i32), C.POINTER(C.c_double), C.POINTER(gsap_stats)]
        L.gsap_create.argtypes = [i32, vp, vp, vp, C.POINTER(gsap_params), C.POINTER(gsap_dist), vp,
                                  C.POINTER(vp)]
        L.gsap_destroy.argtypes = [vp]
        L.gsap_destroy.restype = None
        L.gsap_set_partition.argtypes = [vp, vp, i32]
        L.gsap_get_partition.argtypes = [vp, vp, C.POINTER(i32)]
        L.gsap_update_blockmodel.argtypes = [vp]
        L.gsap_propose.argtypes = [vp, C.c_int, u32, u32, i32, i32, vp]
        L.gsap_delta_mdl.argtypes = [vp, C.c_int, u32, u32, i32, i32, vp, vp, vp, vp]
        L.gsap_select_merges.argtypes = [vp, vp, vp, i32, vp, C.POINTER(i32)]
        L.gsap_apply_moves.argtypes = [vp, i32, i32, vp, vp]
        L.gsap_move_batch.argtypes = [vp, u32, u32, i32, i32, vp, vp, vp, C.POINTER(C.c_double)]
        L.gsap_merge_phase.argtypes = [vp, u32, i32, vp, vp]
        L.gsap_mcmc_phase.argtypes = [vp, u32, C.c_double, vp, C.POINTER(i32)]
        L.gsap_mdl.argtypes = [vp, C.POINTER(C.c_double), C.POINTER(C.c_double)]
        L.gsap_get_blockmodel.argtypes = [vp, i64p] + [vp] * 10
        L.gsap_get_stats.argtypes = [vp, C.POINTER(gsap_stats)]
        L.gsap_reset_stats.argtypes = [vp]
        L.gsap_sync.argtypes = [vp]
        L.gsap_run.argtypes = [vp, vp, C.POINTER(i32), C.POINTER(C.c_double), vp, i32, C.POINTER(i32)]
        L.gsap_nccl_unique_id.argtypes = [vp]
        L.gsap_shard_slice.argtypes = [i32, i32, i32, i32, C.POINTER(i32), C.POINTER(i32), C.POINTER(i32)]
        L.gsap_shard_plan.argtypes = [vp, i32, i32, i32, vp, vp]
        for name in EXPORTED:
            if name not in ("gsap_default_params", "gsap_last_error", "gsap_destroy"):
                getattr(L, name).restype = C.c_int
        _lib = L
    return _lib


def _check(status):
    if status != GSAP_OK:
        raise GsapError(status, lib().gsap_last_error().decode())


def _ptr(x, dtype=None):
    """Raw pointer of a numpy array / torch tensor (None -> NULL).  A CUDA
    tensor is an input the library reads on its own stream (gsap.h): the
    caller's current stream is synchronised first so its producer finished."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        if dtype is not None and x.dtype != dtype:
            raise TypeError(f"expected {np.dtype(dtype)}, got {x.dtype}")
        if not x.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return x.ctypes.data
    import torch
    if isinstance(x, torch.Tensor):
        want = {np.int32: torch.int32, np.int64: torch.int64, np.float64: torch.float64,
                np.uint8: torch.uint8}.get(dtype)
        if want is not None and x.dtype != want:
            raise TypeError(f"expected {want}, got {x.dtype}")
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        if x.is_cuda:
            torch.cuda.current_stream(x.device).synchronize()
        return x.data_ptr()
    raise TypeError(f"unsupported array type {type(x)}")


def _out(n, dtype, device):
    if device:
        import torch
        t = {np.int32: torch.int32, np.int64: torch.int64, np.float64: torch.float64,
             np.uint8: torch.uint8}[dtype]
        return torch.empty(max(n, 0), dtype=t, device="cuda")
    return np.empty(max(n, 0), dtype)


def gsap_default_params(**overrides) -> gsap_params:
    p = gsap_params()
    lib().gsap_default_params(C.byref(p))
    for k, v in overrides.items():
        setattr(p, k, v)
    return p


def gsap_nccl_unique_id() -> bytes:
    """A fresh ncclUniqueId (128 bytes) for gsap_dist; rank 0 creates, the caller broadcasts."""
    buf = (C.c_uint8 * 128)()
    _check(lib().gsap_nccl_unique_id(C.cast(buf, C.c_void_p)))
    return bytes(buf)


def gsap_shard_slice(n, chunk, nranks, rank):
    """(first, count, per_rank) of the slice of [0, n) a rank owns (host only)."""
    f, c, p = C.c_int32(0), C.c_int32(0), C.c_int32(0)
    _check(lib().gsap_shard_slice(n, chunk, nranks, rank, C.byref(f), C.byref(c), C.byref(p)))
    return f.value, c.value, p.value


def make_dist(nranks, rank, device, nccl_id: bytes) -> gsap_dist:
    d = gsap_dist(nranks=nranks, rank=rank, device=device)
    C.memmove(d.nccl_id, nccl_id, 128)
    return d


def dist_from_torch(group=None):
    """gsap_dist for this process from an initialised torch.distributed group."""
    import torch
    import torch.distributed as tdist
    rank, world = tdist.get_rank(group), tdist.get_world_size(group)
    obj = [gsap_nccl_unique_id() if rank == 0 else None]
    tdist.broadcast_object_list(obj, src=0, group=group)
    dev = torch.cuda.current_device() if torch.cuda.is_available() else 0
    return make_dist(world, rank, dev, obj[0])


def gsap_partition(rowptr, col, wgt=None, params=None, device=False, dist=None):
    """One-shot SBP on a CSR digraph; returns dict(b, B, mdl, stats)."""
    rowptr = np.ascontiguousarray(rowptr, np.int64) if isinstance(rowptr, (list, np.ndarray)) else rowptr
    V = int(rowptr.shape[0]) - 1
    params = params or gsap_default_params()
    b = _out(V, np.int32, device)
    B = C.c_int32(0)
    mdl = C.c_double(0)
    st = gsap_stats()
    _check(lib().gsap_partition(V, _ptr(rowptr, np.int64), _ptr(col, np.int32), _ptr(wgt, np.int32),
                                C.byref(params), C.byref(dist) if dist is not None else None, _ptr(b),
                                C.byref(B), C.byref(mdl), C.byref(st)))
    return dict(b=b, B=B.value, mdl=mdl.value, stats=st.as_dict())


class Context:
    """A gsap_ctx: device-resident graph, partition and blockmodel (stepwise API)."""

    def __init__(self, rowptr, col, wgt=None, params=None, stream=None, dist=None):
        self.params = params or gsap_default_params()
        self.V = int(rowptr.shape[0]) - 1
        self._keep = (rowptr, col, wgt)
        h = C.c_void_p()
        _check(lib().gsap_create(self.V, _ptr(rowptr, np.int64), _ptr(col, np.int32),
                                 _ptr(wgt, np.int32), C.byref(self.params),
                                 C.byref(dist) if dist is not None else None, stream, C.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            lib().gsap_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    @property
    def P(self):
        return self.params.num_proposals

    # state ---------------------------------------------------------------
    def gsap_set_partition(self, b, B):
        _check(lib().gsap_set_partition(self.h, _ptr(b, np.int32), int(B)))

    def gsap_get_partition(self, device=False):
        b = _out(self.V, np.int32, device)
        B = C.c_int32(0)
        _check(lib().gsap_get_partition(self.h, _ptr(b), C.byref(B)))
        return b, B.value

    @property
    def B(self):
        B = C.c_int32(0)
        _check(lib().gsap_get_partition(self.h, None, C.byref(B)))
        return B.value

    def gsap_update_blockmodel(self):
        _check(lib().gsap_update_blockmodel(self.h))

    # hot-path steps ------------------------------------------------------
    def gsap_propose(self, phase, outer, itr, first, count, device=False):
        n = count * (self.P if phase == GSAP_MERGE else 1)
        s = _out(n, np.int32, device)
        _check(lib().gsap_propose(self.h, phase, outer, itr, first, count, _ptr(s)))
        return s

    def gsap_delta_mdl(self, phase, outer, itr, first, count, s, device=False):
        n = count * (self.P if phase == GSAP_MERGE else 1)
        dS = _out(n, np.float64, device)
        if phase == GSAP_MOVE:
            H = _out(count, np.float64, device)
            acc = _out(count, np.uint8, device)
            _check(lib().gsap_delta_mdl(self.h, phase, outer, itr, first, count, _ptr(s, np.int32),
                                        _ptr(dS), _ptr(H), _ptr(acc)))
            return dS, H, acc
        _check(lib().gsap_delta_mdl(self.h, phase, outer, itr, first, count, _ptr(s, np.int32),
                                    _ptr(dS), None, None))
        return dS

    def gsap_select_merges(self, best, dS, K, device=False):
        B = self.B
        label = _out(B, np.int32, device)
        nb = C.c_int32(0)
        _check(lib().gsap_select_merges(self.h, _ptr(best, np.int32), _ptr(dS, np.float64), int(K),
                                        _ptr(label), C.byref(nb)))
        return label, nb.value

    def gsap_apply_moves(self, first, count, s, acc):
        _check(lib().gsap_apply_moves(self.h, first, count, _ptr(s, np.int32), _ptr(acc, np.uint8)))

    def gsap_move_batch(self, outer, itr, first, count, outputs=True, device=False):
        s = _out(count, np.int32, device) if outputs else None
        dS = _out(count, np.float64, device) if outputs else None
        acc = _out(count, np.uint8, device) if outputs else None
        dsum = C.c_double(0)
        _check(lib().gsap_move_batch(self.h, outer, itr, first, count, _ptr(s), _ptr(dS), _ptr(acc),
                                     C.byref(dsum)))
        return s, dS, acc, dsum.value

    def gsap_merge_phase(self, outer, K, device=False):
        B = self.B
        best = _out(B, np.int32, device)
        dSb = _out(B, np.float64, device)
        _check(lib().gsap_merge_phase(self.h, outer, int(K), _ptr(best), _ptr(dSb)))
        return best, dSb

    def gsap_mcmc_phase(self, outer, thresh):
        """One MCMC phase from the current state: (iterations run, D[itr] per iteration)."""
        D = np.zeros(self.params.max_nodal_itr + 1)
        n = C.c_int32(0)
        _check(lib().gsap_mcmc_phase(self.h, outer, float(thresh), D.ctypes.data, C.byref(n)))
        return n.value, D[:n.value]

    def gsap_mdl(self):
        m, d = C.c_double(0), C.c_double(0)
        _check(lib().gsap_mdl(self.h, C.byref(m), C.byref(d)))
        return m.value, d.value

    def gsap_get_blockmodel(self):
        nnz = C.c_int64(0)
        _check(lib().gsap_get_blockmodel(self.h, C.byref(nnz), *([None] * 10)))
        n, B = nnz.value, self.B
        out = dict(rowptr=np.zeros(B + 1, np.int64), col=np.zeros(n, np.int32), cnt=np.zeros(n, np.int32),
                   cum=np.zeros(n, np.int32), colptr=np.zeros(B + 1, np.int64), row=np.zeros(n, np.int32),
                   ccnt=np.zeros(n, np.int32), ccum=np.zeros(n, np.int32), dout=np.zeros(B, np.int32),
                   din=np.zeros(B, np.int32))
        _check(lib().gsap_get_blockmodel(self.h, C.byref(nnz), *[_ptr(out[k]) for k in (
            "rowptr", "col", "cnt", "cum", "colptr", "row", "ccnt", "ccum", "dout", "din")]))
        return out

    def gsap_blockmodel_nnz(self):
        """Number of non-zero blockmodel entries (size query of gsap_get_blockmodel)."""
        nnz = C.c_int64(0)
        _check(lib().gsap_get_blockmodel(self.h, C.byref(nnz), *([None] * 10)))
        return nnz.value

    def gsap_shard_plan(self, first, count, nranks):
        """(first[nranks], count[nranks]): the edge-balanced slices of a MOVE batch."""
        f = np.zeros(nranks, np.int32)
        n = np.zeros(nranks, np.int32)
        _check(lib().gsap_shard_plan(self.h, first, count, nranks, f.ctypes.data, n.ctypes.data))
        return f, n

    def gsap_get_stats(self):
        st = gsap_stats()
        _check(lib().gsap_get_stats(self.h, C.byref(st)))
        return st.as_dict()

    def gsap_reset_stats(self):
        _check(lib().gsap_reset_stats(self.h))

    def gsap_sync(self):
        _check(lib().gsap_sync(self.h))

    def gsap_run(self, trace_cap=1024, device=False):
        b = _out(self.V, np.int32, device)
        B = C.c_int32(0)
        mdl = C.c_double(0)
        rounds = C.c_int32(0)
        trace = np.zeros(TRACE_COLS * trace_cap)
        _check(lib().gsap_run(self.h, _ptr(b), C.byref(B), C.byref(mdl), trace.ctypes.data, trace_cap,
                              C.byref(rounds)))
        tr = trace[:TRACE_COLS * min(rounds.value, trace_cap)].reshape(-1, TRACE_COLS)
        return dict(b=b, B=B.value, mdl=mdl.value, trace=tr, rounds=rounds.value)
