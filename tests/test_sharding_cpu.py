"""Multi-rank host logic on CPU (gloo, world_size 2): region sharding has no
data-path collective, and because Philox is keyed by the GLOBAL region id a
region's schedule does not depend on which rank computes it.  The per-rank
compute here is the oracle (test infrastructure), so this checks the
partitioning and gathering logic, not the kernels."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from paper_conf_cgo_shobakimhlmkrg24_b200 import sharding as SH


def test_lpt_partition_covers_and_balances():
    sizes = I.c3_sizes(400, base_seed=3)
    for world in (1, 2, 4, 8):
        parts = SH.lpt_partition(sizes, world)
        flat = sorted(i for p in parts for i in p)
        assert flat == list(range(len(sizes)))
        loads = [sum(SH.estimated_work(int(sizes[i]), 1024, 10) for i in p) for p in parts]
        biggest = max(SH.estimated_work(int(s), 1024, 10) for s in sizes)
        assert max(loads) - min(loads) <= biggest  # LPT bound
        assert parts == SH.lpt_partition(sizes, world)  # deterministic


def test_weak_ids_disjoint():
    a, b = SH.weak_ids(100, 0), SH.weak_ids(100, 1)
    assert not set(a) & set(b) and len(a) == len(b) == 100


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from oracle import pyoracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    regs = I.gen_batch(12, base_seed=21)
    sizes = [r.n_insts for r in regs]
    mine = SH.lpt_partition(sizes, world, ants=32, iterations=2)[rank]
    p = I.Params(ants=32, iterations=2, seed=9)
    local = {}
    for i in mine:
        res = O.schedule(regs[i], i, I.GFX906, p)
        local[i] = {"hash": res["trace_hash"], "len": res["length"], "order": list(map(int, res["order"]))}
    out = SH.gather_results(local, world, rank)
    if rank == 0:
        q.put(out)
    dist.destroy_process_group()


def test_two_rank_gather_equals_single_process():
    from oracle import pyoracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    out = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    regs = I.gen_batch(12, base_seed=21)
    p = I.Params(ants=32, iterations=2, seed=9)
    assert sorted(out) == list(range(12))
    for i, r in enumerate(regs):
        res = O.schedule(r, i, I.GFX906, p)
        assert out[i]["hash"] == res["trace_hash"]
        assert out[i]["order"] == list(map(int, res["order"]))


# ---------------------------------------------------------------- shared colony exchange
def test_colony_key_orders_like_cost_then_ant():
    import random
    rng = random.Random(5)
    pairs = [(rng.choice([0, 1, 7, 23, 0xFFFFFFFE, SH.INVALID_COST]), rng.randrange(0, 1 << 20)) for _ in range(400)]
    for a in pairs:
        assert SH.colony_decode(SH.colony_key(*a)) == a
    for a, b in zip(pairs, pairs[1:]):
        assert (SH.colony_key(*a) < SH.colony_key(*b)) == (a < b)  # signed int64 order == (cost, ant) order


def _colony_worker(rank, world, port, q):
    """One shared-colony rank: its ants are [rank * A_loc, (rank + 1) * A_loc)
    of the global colony; per (region, pass, iteration) it contributes its
    local best key and the MIN all-reduce (gloo here, NCCL on the GPU path)
    must yield the global (cost, ant) minimum on every rank."""
    import torch
    import torch.distributed as dist
    from oracle import pyoracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    regs = [I.fix10a(), I.gen_region(40, 3)]
    p = I.Params(ants=64, iterations=3, seed=11, cost_mode=0)
    a_loc = p.ants // world
    out = []
    for k, r in enumerate(regs):
        cost = O.schedule(r, k, I.GFX906, p, dump=True)["dump_cost"]  # [pass][iter][global ant]
        for ps in range(2):
            for it in range(p.iterations):
                mine = cost[ps, it, rank * a_loc:(rank + 1) * a_loc]
                keys = torch.tensor([SH.local_best_key(list(map(int, mine)), rank * a_loc)], dtype=torch.int64)
                SH.colony_allreduce(keys)
                out.append(SH.colony_decode(int(keys[0])))
    q.put((rank, out))
    dist.destroy_process_group()


def test_two_rank_colony_allreduce_finds_global_winner():
    from oracle import pyoracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_colony_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    got = dict(q.get(timeout=300) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert got[0] == got[1]  # every rank learns the same winner
    regs = [I.fix10a(), I.gen_region(40, 3)]
    p = I.Params(ants=64, iterations=3, seed=11, cost_mode=0)
    want = []
    for k, r in enumerate(regs):
        cost = O.schedule(r, k, I.GFX906, p, dump=True)["dump_cost"]
        for ps in range(2):
            for it in range(p.iterations):
                c = list(map(int, cost[ps, it]))
                a = min(range(len(c)), key=lambda i: (c[i], i))  # R10
                want.append((c[a], a))
    assert got[0] == want
