"""N>1 host logic on CPU (world_size 2, gloo, 127.0.0.1): every rank builds its
owner partition independently from the same edge list; together the partitions
must cover every edge exactly once, with disjoint contiguous owner ranges, and
the activation CSRs must route every edge to the rank owning its destination
(DESIGN.md §10)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import grgen
import paper_conf_sc_senguptasas15_b200 as gr


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = grgen.rmat(12, 16, seed=31)
        H = gr.HostLayout(g.n, g.src, g.dst, world=world, rank=rank, shard_edges=3000)
        lo, hi = int(H.bounds[0]), int(H.bounds[-1])
        meta = torch.tensor([lo, hi, len(H.in_src), len(H.out_dst)], dtype=torch.int64)
        allm = [torch.zeros(4, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allm, meta)
        allm = torch.stack(allm).numpy()
        # CSC payloads gathered to every rank (padded all_gather)
        cap = int(allm[:, 2].max())
        mine = torch.zeros(cap, dtype=torch.int64)
        mine[: len(H.in_src)] = torch.from_numpy(H.in_src.astype(np.int64))
        alls = [torch.zeros(cap, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(alls, mine)
        ok = True
        ok &= allm[0, 0] == 0 and allm[-1, 1] == g.n
        ok &= all(allm[i + 1, 0] == allm[i, 1] for i in range(world - 1))
        ok &= int(allm[:, 2].sum()) == g.m and int(allm[:, 3].sum()) == g.m
        # concatenated per-rank CSCs == the single-rank CSC
        full = gr.HostLayout(g.n, g.src, g.dst)
        cat = np.concatenate([alls[r][: allm[r, 2]].numpy() for r in range(world)])
        ok &= np.array_equal(cat, full.in_src.astype(np.int64))
        # this rank's activation CSR only targets owned vertices, one entry per owned in-edge
        ok &= bool(np.all((H.out_dst >= lo) & (H.out_dst < hi)))
        owned = (g.dst >= lo) & (g.dst < hi)
        ok &= np.array_equal(np.diff(H.out_off.astype(np.int64)), np.bincount(g.src[owned], minlength=g.n))
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def test_two_rank_partition_gloo():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {0: True, 1: True}
