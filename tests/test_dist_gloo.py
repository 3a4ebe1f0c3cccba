"""Multi-GPU host-side logic on CPU (world size 2, gloo): the slicing used by the
sharded MOVE batches and merge phases, the all-gather protocol (each rank
computes its slice, results and fixed-chunk dS partials gathered, applied
identically everywhere) reproducing the single-process run bit for bit, and
the NCCL-id bootstrap over a torch.distributed group.  The compute steps are
the oracle's; the slicing is libgsap's gsap_shard_slice (host function)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from gen import dcsbm

SEED = dcsbm.RUN_SEED
CHUNK = 1024


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_shard_slices_partition_the_range():
    from paper_conf_icpp_changzh24_b200 import gsap
    for n in (0, 1, 250, 1023, 1024, 1025, 5000, 50000, 250001):
        for G in (1, 2, 3, 4, 8):
            pos = 0
            per0 = None
            for g in range(G):
                f, c, per = gsap.gsap_shard_slice(n, CHUNK, G, g)
                per0 = per if per0 is None else per0
                assert per == per0 and per % CHUNK == 0 and per * G >= n
                assert c == 0 or f == g * per            # rank-blocked layout of the all-gather
                assert f == min(pos, n) and c >= 0
                pos = f + c
            assert pos == n


def _protocol(rank, world, port, out):
    from oracle import oracle
    from paper_conf_icpp_changzh24_b200 import gsap
    if world > 1:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    rowptr, col, truth, cfg = dcsbm.make("1k")
    V = cfg.V
    orc = oracle.Oracle(rowptr, col)
    B = 40
    orc.set_partition(dcsbm.random_partition(V, B, 5), B)
    bs = (V + 3) // 4
    record = []
    # a merge phase: every rank proposes for its slice of blocks, winners all-gathered
    f, n, per = gsap.gsap_shard_slice(B, 1, world, rank)
    best = np.zeros(per * world, np.int32)
    dSb = np.zeros(per * world)
    if n:
        s = orc.propose(0, SEED, 0, 0, f, n)
        bo, do = orc.best_merges(s, orc.delta_merge(f, n, s))
        best[f:f + n], dSb[f:f + n] = bo, do
    if world > 1:
        tb, td = torch.from_numpy(best), torch.from_numpy(dSb)
        lb = [torch.zeros_like(tb[:per]) for _ in range(world)]
        ld = [torch.zeros_like(td[:per]) for _ in range(world)]
        dist.all_gather(lb, tb[rank * per:(rank + 1) * per].clone())
        dist.all_gather(ld, td[rank * per:(rank + 1) * per].clone())
        best, dSb = torch.cat(lb).numpy(), torch.cat(ld).numpy()
    orc.select_merges(best[:B], dSb[:B], int(0.4 * B))
    record.append(("merge", orc.partition()[0].tobytes()))
    # MOVE batches: slices of whole chunks; s / acc / chunk partials gathered
    for itr in range(2):
        for k in range(4):
            first, count = k * bs, min(V, (k + 1) * bs) - k * bs
            f, n, per = gsap.gsap_shard_slice(count, CHUNK, world, rank)
            pc = per // CHUNK
            s_buf = np.zeros(per * world, np.int32)
            a_buf = np.zeros(per * world, np.uint8)
            p_buf = np.zeros(pc * world)
            if n:
                s = orc.propose(1, SEED, 1, itr, first + f, n)
                dS, H, p, acc = orc.delta_move(SEED, 1, itr, first + f, n, s)
                s_buf[rank * per:rank * per + n] = s
                a_buf[rank * per:rank * per + n] = acc
                for c in range((n + CHUNK - 1) // CHUNK):
                    sl = slice(c * CHUNK, min(n, (c + 1) * CHUNK))
                    p_buf[rank * pc + c] = float(np.sum(dS[sl][acc[sl] == 1]))
            if world > 1:
                outs = []
                for arr, cnt in ((s_buf, per), (a_buf, per), (p_buf, pc)):
                    t = torch.from_numpy(arr)
                    lst = [torch.zeros_like(t[:cnt]) for _ in range(world)]
                    dist.all_gather(lst, t[rank * cnt:(rank + 1) * cnt].clone())
                    outs.append(torch.cat(lst).numpy())
                s_buf, a_buf, p_buf = outs
            orc.apply_moves(first, count, s_buf[:count], a_buf[:count])
            orc.rebuild()
            chunks = (count + CHUNK - 1) // CHUNK
            D = 0.0
            for c in range(chunks):              # fixed order: identical for any world size
                D += p_buf[c]
            record.append((orc.partition()[0].tobytes(), D))
    out[rank] = record
    if world > 1:
        dist.destroy_process_group()


def test_sharded_protocol_matches_single_process():
    mgr = mp.get_context("spawn").Manager()
    single = mgr.dict()
    _protocol(0, 1, 0, single)
    multi = mgr.dict()
    port = _free_port()
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_protocol, args=(r, 2, port, multi)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    ref = single[0]
    for r in range(2):
        got = multi[r]
        assert len(got) == len(ref)
        for a, b in zip(got, ref):
            assert a == b           # identical partitions and bit-identical D


def _bootstrap(rank, world, port, out):
    from paper_conf_icpp_changzh24_b200 import gsap
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    d = gsap.dist_from_torch()
    out[rank] = (d.nranks, d.rank, bytes(d.nccl_id))
    dist.destroy_process_group()


def test_nccl_id_bootstrap_over_gloo():
    try:
        from paper_conf_icpp_changzh24_b200 import gsap
        gsap.gsap_nccl_unique_id()
    except Exception as e:  # pragma: no cover
        pytest.skip(f"NCCL not loadable: {e}")
    mgr = mp.get_context("spawn").Manager()
    out = mgr.dict()
    port = _free_port()
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_bootstrap, args=(r, 2, port, out)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert out[0][0] == out[1][0] == 2 and {out[0][1], out[1][1]} == {0, 1}
    assert out[0][2] == out[1][2] and len(out[0][2]) == 128
