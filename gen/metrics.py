"""Partition-quality metrics against planted truth (§4.4, Table 4; the
GraphChallenge evaluation): NMI and pairwise precision / recall.  No method
arithmetic; used by tests and bench to compare runs."""
from __future__ import annotations

import numpy as np


def contingency(truth, pred):
    truth = np.asarray(truth, np.int64)
    pred = np.asarray(pred, np.int64)
    _, ti = np.unique(truth, return_inverse=True)
    _, pi = np.unique(pred, return_inverse=True)
    C = np.zeros((ti.max() + 1, pi.max() + 1), np.int64)
    np.add.at(C, (ti, pi), 1)
    return C


def nmi(truth, pred):
    """Normalized mutual information, arithmetic-mean normalisation."""
    C = contingency(truth, pred).astype(np.float64)
    n = C.sum()
    pt = C.sum(1) / n
    pp = C.sum(0) / n
    nz = C > 0
    pij = C[nz] / n
    mi = float(np.sum(pij * np.log(pij / np.outer(pt, pp)[nz])))
    ht = -float(np.sum(pt[pt > 0] * np.log(pt[pt > 0])))
    hp = -float(np.sum(pp[pp > 0] * np.log(pp[pp > 0])))
    if ht + hp == 0:
        return 1.0
    return 2.0 * mi / (ht + hp)


def pairwise_precision_recall(truth, pred):
    """Over all vertex pairs: precision = P(same truth | same pred), recall =
    P(same pred | same truth) (GraphChallenge pairwise metrics)."""
    C = contingency(truth, pred)
    both = int(np.sum(C * (C - 1) // 2))
    same_pred = int(np.sum(C.sum(0) * (C.sum(0) - 1) // 2))
    same_truth = int(np.sum(C.sum(1) * (C.sum(1) - 1) // 2))
    prec = both / same_pred if same_pred else 1.0
    rec = both / same_truth if same_truth else 1.0
    return prec, rec


def load_tsv(path, one_based=True):
    """GraphChallenge TSV edge list (src dst [weight]) -> (rowptr int64, col int32, wgt int32|None).
    Ids are 1-based in the challenge files."""
    a = np.loadtxt(path, dtype=np.int64, ndmin=2)
    src, dst = a[:, 0], a[:, 1]
    if one_based:
        src, dst = src - 1, dst - 1
    V = int(max(src.max(), dst.max()) + 1) if len(a) else 0
    w = a[:, 2].astype(np.int32) if a.shape[1] > 2 else None
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    rowptr = np.zeros(V + 1, np.int64)
    np.add.at(rowptr, src + 1, 1)
    rowptr = np.cumsum(rowptr)
    return rowptr, dst.astype(np.int32), (None if w is None else w[order])


def load_truth_tsv(path, V, one_based=True):
    """GraphChallenge truth file (vertex block) -> int32[V]."""
    a = np.loadtxt(path, dtype=np.int64, ndmin=2)
    t = np.full(V, -1, np.int64)
    t[a[:, 0] - (1 if one_based else 0)] = a[:, 1] - (1 if one_based else 0)
    return t.astype(np.int32)
