"""Multi-process host logic of the N>1 path on CPU (gloo, world size 2): the record
sharding of bench ranks, the NCCL unique-id broadcast used to build the merge
communicator, and the max-over-ranks timing reduction.  The device side of the
rank merge is covered on one GPU by test_gpu_parity.test_rank_merge_simulated."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_zhouhmm022_b200 import ve
        import bench
        # 1. sharding: contiguous, disjoint, covering -- gathered from every rank
        n = 231555071
        lo, hi = ve.rank_chunk(n, rank, world)
        t = torch.tensor([lo, hi], dtype=torch.int64)
        allc = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allc, t)
        # 2. the unique-id broadcast of nccl_comm_from_torch (bytes identical on every rank)
        uid = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            uid = torch.arange(128, dtype=torch.uint8) ^ 0x5A
        dist.broadcast(uid, src=0)
        ids = [torch.zeros(128, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(ids, uid)
        # 3. the max-over-ranks timing reduction of bench.py
        ms = bench.max_over_ranks(10.0 + rank, device="cpu")
        # 4. cfg5's kernel plan (LPT on record count), computed independently on every rank
        from gen import vegen as G
        cfg = G.scaled(G.CFG5, 0)
        costs = [G.info(cfg, k)["n_records"] for k in range(4000)]
        owner = ve.lpt_assign(costs, world)
        mine = [k for k in range(4000) if owner[k] == rank]
        t = torch.tensor([len(mine), sum(costs[k] for k in mine), sum(mine), hash(tuple(owner)) & 0x7FFFFFFF],
                         dtype=torch.int64)
        plans = [torch.zeros(4, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(plans, t)
        q.put((rank, [c.tolist() for c in allc], [bytes(i.tolist()) for i in ids], ms, [p.tolist() for p in plans]))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n = 231555071
    for rank, chunks, ids, ms, plans in res:
        # the kernel plan: the same on both ranks, covering every kernel once, balanced
        assert len({p[3] for p in plans}) == 1
        assert sum(p[0] for p in plans) == 4000 and sum(p[2] for p in plans) == 4000 * 3999 // 2
        assert sum(p[1] for p in plans) == 1_000_000_000
        loads = [p[1] for p in plans]
        assert max(loads) <= (4 / 3 - 1 / (3 * world)) * max(1_000_000_000 / world, 1_676_166)
        assert chunks[0][0] == 0 and chunks[-1][1] == n
        assert all(chunks[i][1] == chunks[i + 1][0] for i in range(world - 1))
        assert len(set(ids)) == 1 and ids[0] == bytes((i ^ 0x5A) for i in range(128))
        assert ms == 11.0


def test_lpt_assign_bound():
    """LPT against the brute-force optimum on small random instances: every unit assigned,
    max load within Graham's (4/3 - 1/(3m)) bound, deterministic."""
    import itertools
    import random
    from paper_conf_asplos_zhouhmm022_b200 import ve
    rng = random.Random(5)
    for _ in range(40):
        m = rng.choice([2, 3])
        costs = [rng.randint(1, 50) for _ in range(rng.randint(1, 8))]
        owner = ve.lpt_assign(costs, m)
        assert owner == ve.lpt_assign(list(costs), m) and all(0 <= r < m for r in owner)
        loads = [sum(c for c, r in zip(costs, owner) if r == q) for q in range(m)]
        opt = min(max(sum(c for c, r in zip(costs, a) if r == q) for q in range(m))
                  for a in itertools.product(range(m), repeat=len(costs)))
        assert max(loads) <= (4 / 3 - 1 / (3 * m)) * opt + 1e-9
