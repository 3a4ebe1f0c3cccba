"""Seeded synthetic inputs: GraphChallenge-shaped degree-corrected SBM digraphs.

This module holds NO arithmetic of the partitioning method.  It only draws
graphs (and the seeds the runs use), and serves both the CUDA path and the CPU
oracle.  Recipe (PAPER.md P:75-110
§2.2 Table 1; Karrer & Newman [45] P:455):

* planted block count B = floor(V**0.35) (reproduces every Table 1 B),
* block shares pi ~ Dirichlet(alpha * 1): alpha = 10 (low size variation) or
  alpha = 1 (high size variation); block sizes ~ Multinomial(V, pi), each >= 1,
  vertex ids randomly permuted,
* within-block edge fraction omega = rho / (1 + rho): rho = 5 (low overlap) or
  rho = 2.5 (high overlap),
* lambda_rs = E [omega d_rs s_r + (1 - omega)(1 - d_rs) s_r s_s / (1 - sum s^2)]
  with s the realised block shares; M_rs ~ Poisson(lambda_rs),
* endpoints within a block proportional to theta_out / theta_in, theta i.i.d.
  from the truncated power law p(theta) ~ theta^-2.5 on [1, 100],
* duplicate (u, v) pairs collapsed to unit weight, self-loops kept, then a
  seeded subsample to exactly the Table 1 edge count.
"""
from __future__ import annotations

import dataclasses

import numpy as np


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    V: int
    E: int
    alpha: float
    rho: float

    @property
    def B_planted(self) -> int:
        return int(np.floor(self.V ** 0.35 + 1e-9))


# BASELINE.json configs (Table 1 shapes)
CONFIGS = {
    "1k": Config("1K-LL", 1_000, 8_067, 10.0, 5.0),
    "20k": Config("20K-HH", 20_000, 473_329, 1.0, 2.5),
    "200k": Config("200K-HL", 200_000, 4_743_468, 10.0, 2.5),
    "1m": Config("1M-LL", 1_000_000, 23_716_108, 10.0, 5.0),
    "2m": Config("2M-LL", 2_000_000, 47_432_216, 10.0, 5.0),
}

RUN_SEED = 0x5B9D2024


def _theta(rng, n, lo=1.0, hi=100.0, a=2.5):
    # inverse CDF of p(x) ~ x^-a on [lo, hi]
    u = rng.random(n)
    e = 1.0 - a
    return (lo ** e + u * (hi ** e - lo ** e)) ** (1.0 / e)


def _within(rng, block_of_edge, starts, cum_w, order):
    """Pick one vertex per edge inside its block, proportional to weights."""
    u = rng.random(len(block_of_edge))
    lo = starts[block_of_edge]
    base = np.where(lo > 0, cum_w[np.maximum(lo - 1, 0)], 0.0)
    tot = cum_w[starts[block_of_edge + 1] - 1] - base
    tgt = base + u * tot
    idx = np.searchsorted(cum_w, tgt, side="right")
    idx = np.minimum(np.maximum(idx, lo), starts[block_of_edge + 1] - 1)
    return order[idx]


def _sorted_unique(a):
    # == np.unique(a) (sorted distinct values); numpy 2.3's hash-based unique is ~5x slower here
    a = np.sort(a)
    if len(a) == 0:
        return a
    keep = np.empty(len(a), bool)
    keep[0] = True
    np.not_equal(a[1:], a[:-1], out=keep[1:])
    return a[keep]


def generate(V: int, E: int, alpha: float, rho: float, seed: int | None = None,
             B: int | None = None):
    """Return (rowptr int64[V+1], col int32[E], truth int32[V]); CSR rows sorted."""
    seed = V if seed is None else seed
    rng = np.random.default_rng(seed)
    B = int(np.floor(V ** 0.35 + 1e-9)) if B is None else B
    B = max(1, min(B, V))
    pi = rng.dirichlet(np.full(B, alpha))
    sizes = rng.multinomial(V - B, pi) + 1
    truth = np.repeat(np.arange(B, dtype=np.int32), sizes)
    truth = truth[rng.permutation(V)]
    th_out = _theta(rng, V)
    th_in = _theta(rng, V)
    order = np.argsort(truth, kind="stable")          # vertices grouped by block
    starts = np.zeros(B + 1, np.int64)
    starts[1:] = np.cumsum(sizes)
    cum_out = np.cumsum(th_out[order])
    cum_in = np.cumsum(th_in[order])
    share = sizes / V
    omega = rho / (1.0 + rho)
    denom = max(1.0 - float(np.sum(share ** 2)), 1e-12)
    want = E
    edges = np.zeros(0, np.int64)
    scale = 1.0
    for _ in range(8):
        lam = (1 - omega) * np.outer(share, share) / denom
        np.fill_diagonal(lam, omega * share)
        lam *= want * scale
        cnt = rng.poisson(lam).ravel()
        pairs = np.repeat(np.arange(B * B, dtype=np.int64), cnt)
        src_b = pairs // B
        dst_b = pairs % B
        src = _within(rng, src_b, starts, cum_out, order)
        dst = _within(rng, dst_b, starts, cum_in, order)
        edges = _sorted_unique(np.concatenate([edges, src.astype(np.int64) * V + dst]))
        if len(edges) >= E:
            break
        scale = max(0.05, (E - len(edges)) / max(want, 1) * 1.1)
    if len(edges) > E:
        keep = np.sort(rng.choice(len(edges), E, replace=False))
        edges = edges[keep]
    src = (edges // V).astype(np.int64)
    col = (edges % V).astype(np.int32)
    rowptr = np.zeros(V + 1, np.int64)
    rowptr[1:] = np.bincount(src, minlength=V)
    rowptr = np.cumsum(rowptr)
    return rowptr, col, truth.astype(np.int32)


def make(name: str):
    """The named BASELINE.json config: (rowptr, col, truth, Config)."""
    c = CONFIGS[name]
    rowptr, col, truth = generate(c.V, c.E, c.alpha, c.rho, seed=c.V)
    return rowptr, col, truth, c


def random_multigraph(V, E, seed, self_loops=True, weighted=False, max_w=5):
    """Tiny random multigraph (duplicates and self-loops allowed) for pins."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, V, E)
    dst = rng.integers(0, V, E)
    if not self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    order = np.argsort(src, kind="stable")
    src, dst = src[order], dst[order]
    rowptr = np.zeros(V + 1, np.int64)
    np.add.at(rowptr, src + 1, 1)
    rowptr = np.cumsum(rowptr)
    w = rng.integers(1, max_w + 1, len(dst)).astype(np.int32) if weighted else None
    return rowptr, dst.astype(np.int32), w


def random_partition(V, B, seed):
    rng = np.random.default_rng(seed)
    b = rng.integers(0, B, V).astype(np.int32)
    b[:min(B, V)] = np.arange(min(B, V), dtype=np.int32)[:V]  # every block non-empty
    return b[rng.permutation(V)] if V > 1 else b
