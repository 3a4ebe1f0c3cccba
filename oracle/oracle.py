"""ctypes wrapper of the CPU oracle (oracle/gsap_oracle.c).

TEST INFRASTRUCTURE, NOT PART OF THE PRODUCT PATH.  Only tests/,
``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl
reference`` leg may import this module.  It never imports the product package
and the product package never imports it.

The oracle is a plain, slow, obviously-correct C implementation of the GSAP
hot path written from /root/reference/PAPER.md; see the header of
gsap_oracle.c and DESIGN.md ("Oracle").
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "gsap_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

_i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")
_u8p = np.ctypeslib.ndpointer(np.uint8, flags="C_CONTIGUOUS")
_u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")


class OParams(C.Structure):
    _fields_ = [
        ("seed", C.c_uint64),
        ("beta", C.c_double),
        ("reduction_rate", C.c_double),
        ("num_proposals", C.c_int32),
        ("max_nodal_itr", C.c_int32),
        ("thresh1", C.c_double),
        ("thresh2", C.c_double),
        ("window", C.c_int32),
        ("num_batches", C.c_int32),
        ("model_term", C.c_int32),
        ("max_rounds", C.c_int32),
    ]


class OStats(C.Structure):
    _fields_ = [
        ("n_move_prop", C.c_int64),
        ("n_move_acc", C.c_int64),
        ("n_merge_prop", C.c_int64),
        ("rounds", C.c_int32),
        ("mcmc_itr_total", C.c_int32),
    ]


def default_params(**kw) -> OParams:
    """Table 2 (§4.1) + readings Z3-Z5."""
    p = OParams(seed=0x5B9D2024, beta=3.0, reduction_rate=0.4, num_proposals=10,
                max_nodal_itr=100, thresh1=5e-4, thresh2=1e-4, window=3,
                num_batches=4, model_term=0, max_rounds=500)
    for k, v in kw.items():
        setattr(p, k, v)
    return p


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2, strict IEEE, x87 long double)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-fopenmp",
                               "-o", LIB, SRC, "-lm"])
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        L.orc_philox.argtypes = [_u32p, _u32p, _u32p]
        L.orc_set_threads.restype = C.c_int32
        L.orc_set_threads.argtypes = [C.c_int32]
        L.orc_set_proposal_mode.argtypes = [C.c_void_p, C.c_int]
        L.orc_table.argtypes = [C.c_void_p, C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, _i32p]
        L.orc_create.restype = C.c_void_p
        L.orc_create.argtypes = [C.c_int32, _i64p, _i32p, C.c_void_p]
        L.orc_destroy.argtypes = [C.c_void_p]
        L.orc_set_partition.argtypes = [C.c_void_p, _i32p, C.c_int32]
        L.orc_set_b_norebuild.argtypes = [C.c_void_p, _i32p, C.c_int32]
        L.orc_get_partition.restype = C.c_int32
        L.orc_get_partition.argtypes = [C.c_void_p, _i32p]
        L.orc_rebuild.argtypes = [C.c_void_p]
        L.orc_nnz.restype = C.c_int64
        L.orc_nnz.argtypes = [C.c_void_p]
        L.orc_total_weight.restype = C.c_int64
        L.orc_total_weight.argtypes = [C.c_void_p]
        L.orc_get_blockmodel.argtypes = [C.c_void_p] + [C.c_void_p] * 10
        L.orc_mdl.restype = C.c_double
        L.orc_mdl.argtypes = [C.c_void_p, C.c_int, C.POINTER(C.c_double)]
        L.orc_propose.argtypes = [C.c_void_p, C.c_int, C.c_uint64, C.c_uint32, C.c_uint32,
                                  C.c_int32, C.c_int32, C.c_int32, _i32p]
        L.orc_delta_move.argtypes = [C.c_void_p, C.c_uint64, C.c_uint32, C.c_uint32, C.c_double,
                                     C.c_int32, C.c_int32, _i32p, _f64p, _f64p, _f64p, _u8p]
        L.orc_delta_merge.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, _i32p, _f64p]
        L.orc_best_merges.argtypes = [C.c_int32, C.c_int32, _i32p, _f64p, _i32p, _f64p]
        L.orc_select_merges.restype = C.c_int32
        L.orc_select_merges.argtypes = [C.c_void_p, _i32p, _f64p, C.c_int32, C.c_void_p]
        L.orc_apply_moves.argtypes = [C.c_void_p, C.c_int32, C.c_int32, _i32p, _u8p]
        L.orc_partition.restype = C.c_int32
        L.orc_partition.argtypes = [C.c_void_p, C.POINTER(OParams), _i32p, C.POINTER(C.c_int32),
                                    C.POINTER(C.c_double), C.POINTER(OStats), _f64p, C.c_int32]
        L.orc_mcmc_phase.restype = C.c_int32
        L.orc_mcmc_phase.argtypes = [C.c_void_p, C.POINTER(OParams), C.c_uint32, C.c_double,
                                     C.POINTER(OStats), C.c_void_p]
        L.orc_mcmc_stop_mock.restype = C.c_int32
        L.orc_mcmc_stop_mock.argtypes = [_f64p, _f64p, C.c_int32, C.c_int32, C.c_double]
        L.orc_merge_phase.restype = C.c_int32
        L.orc_merge_phase.argtypes = [C.c_void_p, C.POINTER(OParams), C.c_uint32, C.c_int32]
        L.orc_mcmc_batch.restype = C.c_double
        L.orc_mcmc_batch.argtypes = [C.c_void_p, C.POINTER(OParams), C.c_uint32, C.c_uint32,
                                     C.c_int32, C.c_int32]
        L.orc_bracket_replay.restype = C.c_int32
        L.orc_bracket_replay.argtypes = [C.c_int32, _i32p, _f64p, C.c_double, _i32p, _i32p, _i32p]
        L.orc_golden_mock.restype = C.c_int32
        L.orc_golden_mock.argtypes = [C.c_int32, C.c_double, _f64p, _i32p, C.c_int32,
                                      C.POINTER(C.c_int32)]
        _lib = L
    return _lib


# orc_partition trace row: [outer, B after merge, MCMC iterations, MDL, threshold used, accepted moves]
TRACE_COLS = 6


def mcmc_stop_mock(D, mdl, window=3, thresh=5e-4):
    """The MCMC stopping rule alone (the helper mcmc_phase calls) against given
    per-iteration D[itr] and MDL[itr] (MDL of the state after iteration itr):
    the number of iterations the phase would run."""
    D = np.ascontiguousarray(D, np.float64)
    mdl = np.ascontiguousarray(mdl, np.float64)
    assert len(D) == len(mdl)
    return lib().orc_mcmc_stop_mock(D, mdl, len(D), window, thresh)


def bracket_replay(B_after_merge, mdl, rate=0.4):
    """The golden-section bracket logic (O.9) replayed over given rounds:
    per round the next round's starting B, its K and whether the bracket is
    established (next round on thresh2); and the number of rounds run."""
    Bs = np.ascontiguousarray(B_after_merge, np.int32)
    S = np.ascontiguousarray(mdl, np.float64)
    n = len(Bs)
    Bn = np.zeros(max(n, 1), np.int32)
    Kn = np.zeros(max(n, 1), np.int32)
    Br = np.zeros(max(n, 1), np.int32)
    stop = lib().orc_bracket_replay(n, Bs, S, rate, Bn, Kn, Br)
    return Bn[:n], Kn[:n], Br[:n].astype(bool), stop


def set_threads(n: int) -> int:
    """OpenMP threads of the oracle's per-id loops (1 = canonical single-thread;
    results are identical for any n).  Returns the number in effect."""
    return lib().orc_set_threads(int(n))


def golden_mock(V, rate, mdl_of_B, cap=1000):
    """Run only the golden-section bracket logic against a table MDL(B)."""
    vis = np.zeros(cap, np.int32)
    Bf = C.c_int32(0)
    n = lib().orc_golden_mock(V, rate, np.ascontiguousarray(mdl_of_B, np.float64), vis, cap,
                              C.byref(Bf))
    return vis[:n], Bf.value


def philox(ctr, key):
    out = np.zeros(4, np.uint32)
    lib().orc_philox(np.asarray(ctr, np.uint32), np.asarray(key, np.uint32), out)
    return out


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class Oracle:
    """One oracle state: graph + partition b + blockmodel (rebuilt from b)."""

    def __init__(self, rowptr, col, wgt=None):
        self.rowptr = np.ascontiguousarray(rowptr, np.int64)
        self.col = np.ascontiguousarray(col, np.int32)
        self.wgt = None if wgt is None else np.ascontiguousarray(wgt, np.int32)
        self.V = len(self.rowptr) - 1
        self.h = lib().orc_create(self.V, self.rowptr, self.col, _ptr(self.wgt))

    def close(self):
        if self.h:
            lib().orc_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # state -----------------------------------------------------------------
    def set_partition(self, b, B):
        lib().orc_set_partition(self.h, np.ascontiguousarray(b, np.int32), int(B))

    def set_proposal_mode(self, mode):
        """N4 ablation: 0 = fresh Philox draws (default), 1 = the paper's shared lookup table."""
        lib().orc_set_proposal_mode(self.h, int(mode))

    def table(self, seed, j, itr, outer, phase):
        """The shared neighbour-block table (N4) for one merge phase / MOVE batch."""
        out = np.zeros(max(self.B, 1), np.int32)
        lib().orc_table(self.h, seed, j, itr, outer, phase, out)
        return out[:self.B]

    def set_b_norebuild(self, b, B):
        lib().orc_set_b_norebuild(self.h, np.ascontiguousarray(b, np.int32), int(B))

    def rebuild(self):
        lib().orc_rebuild(self.h)

    def partition(self):
        b = np.zeros(self.V, np.int32)
        B = lib().orc_get_partition(self.h, b)
        return b, B

    @property
    def B(self):
        return lib().orc_get_partition(self.h, np.zeros(max(self.V, 1), np.int32))

    @property
    def total_weight(self):
        return lib().orc_total_weight(self.h)

    def blockmodel(self):
        """dict of rowptr, col, cnt, cum (CSR), colptr, row, ccnt, ccum (CSC), dout, din."""
        nnz = lib().orc_nnz(self.h)
        B = self.B
        out = dict(rowptr=np.zeros(B + 1, np.int64), col=np.zeros(nnz, np.int32),
                   cnt=np.zeros(nnz, np.int64), cum=np.zeros(nnz, np.int64),
                   colptr=np.zeros(B + 1, np.int64), row=np.zeros(nnz, np.int32),
                   ccnt=np.zeros(nnz, np.int64), ccum=np.zeros(nnz, np.int64),
                   dout=np.zeros(B, np.int64), din=np.zeros(B, np.int64))
        lib().orc_get_blockmodel(self.h, *[_ptr(out[k]) for k in
                                           ("rowptr", "col", "cnt", "cum", "colptr", "row",
                                            "ccnt", "ccum", "dout", "din")])
        return out

    def mdl(self, model_term=0):
        d = C.c_double(0)
        m = lib().orc_mdl(self.h, model_term, C.byref(d))
        return m, d.value

    # hot-path steps --------------------------------------------------------
    def propose(self, phase, seed, outer, itr, first, count, P=10):
        n = count * (P if phase == 0 else 1)
        s = np.zeros(max(n, 1), np.int32)
        lib().orc_propose(self.h, phase, seed, outer, itr, first, count, P, s)
        return s[:n]

    def delta_move(self, seed, outer, itr, first, count, s, beta=3.0):
        s = np.ascontiguousarray(s, np.int32)
        n = max(count, 1)
        dS, H, p = np.zeros(n), np.zeros(n), np.zeros(n)
        acc = np.zeros(n, np.uint8)
        lib().orc_delta_move(self.h, seed, outer, itr, beta, first, count, s, dS, H, p, acc)
        return dS[:count], H[:count], p[:count], acc[:count]

    def delta_merge(self, first, count, s, P=10):
        s = np.ascontiguousarray(s, np.int32)
        dS = np.zeros(max(count * P, 1))
        lib().orc_delta_merge(self.h, first, count, P, s, dS)
        return dS[:count * P]

    @staticmethod
    def best_merges(s, dS, P=10):
        s = np.ascontiguousarray(s, np.int32)
        dS = np.ascontiguousarray(dS, np.float64)
        n = len(s) // P
        best = np.zeros(max(n, 1), np.int32)
        dSb = np.zeros(max(n, 1))
        lib().orc_best_merges(n, P, s, dS, best, dSb)
        return best[:n], dSb[:n]

    def select_merges(self, best, dSbest, K):
        B = self.B
        label = np.zeros(max(B, 1), np.int32)
        newB = lib().orc_select_merges(self.h, np.ascontiguousarray(best, np.int32),
                                       np.ascontiguousarray(dSbest, np.float64), int(K),
                                       _ptr(label))
        return label[:B], newB

    def apply_moves(self, first, count, s, acc):
        lib().orc_apply_moves(self.h, first, count, np.ascontiguousarray(s, np.int32),
                              np.ascontiguousarray(acc, np.uint8))

    def mcmc_batch(self, params, outer, itr, first, count):
        return lib().orc_mcmc_batch(self.h, C.byref(params), outer, itr, first, count)

    def mcmc_phase(self, params, outer, thresh, return_D=False):
        """One MCMC phase (O.8).  return_D: also D[itr] (sum of accepted dS per iteration)."""
        st = OStats()
        D = np.zeros(params.max_nodal_itr + 1)
        n = lib().orc_mcmc_phase(self.h, C.byref(params), outer, thresh, C.byref(st), _ptr(D))
        if return_D:
            return n, st, D[:n]
        return n, st

    def merge_phase(self, params, outer, K):
        return lib().orc_merge_phase(self.h, C.byref(params), outer, int(K))

    def partition_run(self, params=None, trace_cap=1024):
        params = params or default_params()
        b = np.zeros(max(self.V, 1), np.int32)
        B = C.c_int32(0)
        mdl = C.c_double(0)
        st = OStats()
        trace = np.zeros(TRACE_COLS * trace_cap)
        rounds = lib().orc_partition(self.h, C.byref(params), b, C.byref(B), C.byref(mdl),
                                     C.byref(st), trace, trace_cap)
        tr = trace[:TRACE_COLS * min(rounds, trace_cap)].reshape(-1, TRACE_COLS)
        return dict(b=b[:self.V], B=B.value, mdl=mdl.value, stats=st, trace=tr, rounds=rounds)
