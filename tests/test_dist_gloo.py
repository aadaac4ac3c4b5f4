"""N > 1 host logic on CPU with gloo, world size 2.

Each rank takes its row range from the library's ``glp_partition`` (through
``paper_conf_sigmod_yelhls21_b200.dist``), computes its rows' MFL with the
oracle's single-iteration function, exchanges labels with an all-gather and
the stop-rule counters with an all-reduce -- the same protocol libglp.so runs
over NCCL.  Synchronous LP is partition-independent, so every rank must end
with exactly the single-process oracle's labels and iteration count.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from glp_inputs import graphs


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sigmod_yelhls21_b200 import dist as gdist
        name, variant, gamma, edge_balanced = case
        if name == "rmat":
            csr = graphs.rmat(11, seed=4)
            seeds = None
        else:
            csr, seeds = graphs.taobao(users=4000, items=1000, pairs=20000, rings=10, seed=2)
            seeds = seeds.numpy()
        n = csr.n
        bounds = gdist.shard_bounds(n, world, csr.row_offsets, edge_balanced)
        vb, ve = bounds[rank], bounds[rank + 1]
        off_l, col_l = gdist.local_rows(csr.row_offsets, csr.col_idx, vb, ve)
        # the owned rows are exactly the global rows, rebased
        assert off_l[0] == 0 and int(off_l[-1]) == col_l.numel()
        L = oracle.init_labels(n, variant, seeds)
        is_seed = None
        if variant == oracle.SEEDED:
            is_seed = np.zeros(n, dtype=np.uint8)
            is_seed[seeds] = 1
        prev2 = None
        iters, reason = 0, 0
        for t in range(1, 21):
            V = np.bincount(L[L >= 0], minlength=n).astype(np.int32) if variant == oracle.LLP else None
            nxt = oracle.step(csr, variant, L, vb, ve, V=V, is_seed=is_seed, gamma=gamma)
            # exchange: every rank contributes its owned slice (the all-gather)
            mine = torch.from_numpy(nxt[vb:ve].copy())
            sizes = [bounds[r + 1] - bounds[r] for r in range(world)]
            parts = [torch.empty(sz, dtype=torch.int32) for sz in sizes]
            dist.all_gather(parts, mine) if len(set(sizes)) == 1 else _gather_uneven(parts, mine, rank, world)
            full = torch.cat(parts).numpy()
            # stop rule counters: per-rank counts over owned rows, summed
            cnt = torch.tensor([int((full[vb:ve] != L[vb:ve]).sum()),
                                int((full[vb:ve] != prev2[vb:ve]).sum()) if prev2 is not None else 1],
                               dtype=torch.int64)
            dist.all_reduce(cnt)
            prev2, L = L, full
            iters = t
            if cnt[0] == 0:
                reason = 1
                break
            if t >= 2 and cnt[1] == 0:
                reason = 2
                break
        ref = oracle.run(csr, variant, 20, seeds=seeds, gamma=gamma)
        ok = (L == ref.labels).all() and iters == ref.iterations and reason == ref.stop_reason
        q.put((rank, bool(ok), bounds))
    finally:
        dist.destroy_process_group()


def _gather_uneven(parts, mine, rank, world):
    # gloo all_gather needs equal sizes: pad to the max, then trim
    m = max(p.numel() for p in parts)
    padded = torch.full((m,), -7, dtype=torch.int32)
    padded[:mine.numel()] = mine
    outs = [torch.empty(m, dtype=torch.int32) for _ in range(world)]
    dist.all_gather(outs, padded)
    for r in range(world):
        parts[r].copy_(outs[r][:parts[r].numel()])


@pytest.mark.parametrize("case", [("rmat", oracle.CLASSIC, 0.0, False), ("rmat", oracle.LLP, 1.0, True),
                                  ("taobao", oracle.SEEDED, 0.0, False)])
def test_two_rank_partition_matches_single_process(case):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok, _ in res), res
    b0, b1 = res[0][2], res[1][2]
    assert b0 == b1 and b0[0] == 0
