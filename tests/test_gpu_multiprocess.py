"""Two real processes (ranks) on cuda:0 with torch.distributed (gloo on CUDA
tensors; the driver's single-GPU box stands in for two NVLink peers): the
LPT-partitioned region batch (config 3's strong-scaling split, PAPER.md L425
future work) and the shared colony (config 4) through Scheduler.run_colony.
Both equal the one-process run and the oracle bit for bit."""
import os
import socket

import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I

pytestmark = pytest.mark.gpu

KEYS = ("length", "prp", "cost_rp", "iters1", "iters2", "best1", "best2", "init1", "init2", "trace_hash")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _digest(r):
    d = {k: r[k] for k in KEYS}
    d["order"] = [int(x) for x in r["order"]]
    d["cycle"] = [int(x) for x in r["cycle"]]
    return d


def _cmp(d, ora, ctx):
    for k in KEYS:
        assert d[k] == ora[k], (ctx, k)
    assert d["order"] == [int(x) for x in ora["order"]], ctx
    assert d["cycle"] == [int(x) for x in ora["cycle"]], ctx


def _batch():
    sizes = I.c3_sizes(24, 3)
    return sizes, I.gen_regions(range(24), sizes, 3)


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    from paper_conf_cgo_shobakimhlmkrg24_b200 import sharding
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    # (a) partitioned batch: this rank's LPT share, global ids
    sizes, regs = _batch()
    p = I.Params(ants=256, iterations=3, seed=3)
    part = sharding.lpt_partition(sizes, world, p.ants, p.iterations)[rank]
    s = Scheduler(I.GFX906, device=0)
    s.load([regs[i] for i in part], part).run(p)
    local = {i: _digest(r) for i, r in zip(part, s.results())}
    gathered = sharding.gather_results(local, world, rank)
    # (b) shared colony: 2 x 96 ants of two regions (one global-state)
    creg = [I.gen_region(140, 9600), I.gen_region(1300, 9601)]
    pc = I.Params(ants=96, iterations=3, seed=9)
    c = Scheduler(I.GFX906, device=0)
    c.load(creg, [0, 1]).run_colony(pc, rank, world)
    colony = [_digest(r) for r in c.results()]
    torch.cuda.synchronize()
    q.put((rank, gathered, colony))
    dist.barrier()
    dist.destroy_process_group()


def test_two_processes_partitioned_batch_and_colony():
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    out = {}
    for _ in range(2):
        rank, gathered, colony = q.get(timeout=600)
        out[rank] = (gathered, colony)
    for pr in procs:
        pr.join(timeout=120)
        assert pr.exitcode == 0
    # one process, the whole batch
    sizes, regs = _batch()
    p = I.Params(ants=256, iterations=3, seed=3)
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, list(range(24))).run(p)
    single = {i: _digest(r) for i, r in enumerate(s.results())}
    gathered = out[0][0]
    assert sorted(gathered) == list(range(24))
    for i in range(24):
        assert gathered[i] == single[i], i
    for i in (0, 7, 23):
        _cmp(gathered[i], O.schedule(regs[i], i, I.GFX906, p), f"region {i}")
    # colony: both ranks hold identical results == one context with 192 ants == the oracle
    creg = [I.gen_region(140, 9600), I.gen_region(1300, 9601)]
    pc_all = I.Params(ants=192, iterations=3, seed=9)
    for k in range(2):
        assert out[0][1][k] == out[1][1][k], k
        ora = O.schedule(creg[k], k, I.GFX906, pc_all)
        _cmp(out[0][1][k], ora, f"colony region {k}")
