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
