"""Small runs of the CUDA path for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): SAN_CASE = c1 (FIX10-A, 64 ants x 20 iterations), c2
(the config-2 region, 1024 ants x 2 iterations), rl (pass-1 ready-list limit
R45 lockstep, 4 regions incl. a 4-wide one, 128 ants x 2 iterations), gs (a
global-state region, 64 ants x 1 iteration), lean (large regions, lean pass-2
layout), dump (every-ant dump mode), colony (2 emulated ranks).  Each run is
checked against the oracle so a sanitizer pass is also a parity pass."""
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from oracle import pyoracle as O  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

case = os.environ.get("SAN_CASE", "c1")
kw = {}
if case == "c1":
    regs, p = [I.fix10a()], I.Params(ants=64, iterations=20, seed=0, cost_mode=0)
elif case == "c2":
    regs, p = [I.gen_region(100, I.region_seed(2, 0))], I.Params(ants=1024, iterations=2, seed=2)
elif case == "rl":
    regs = [I.fix10a(), I.gen_region(45, 1801), I.gen_region(130, 1802, "unit"), I.gen_region(230, 1803)]
    p = I.Params(ants=128, iterations=2, seed=41, cost_mode=0, rl_limit=1)
elif case == "gs":
    regs, p = [I.gen_region(1300, 9301)], I.Params(ants=64, iterations=1, seed=12)
elif case == "lean":
    regs, p = [I.gen_region(n, 1600 + n) for n in (170, 330, 480)], I.Params(ants=128, iterations=2, seed=24)
elif case == "dump":
    regs, p = [I.gen_region(n, 500 + n) for n in (5, 40, 130)], I.Params(ants=70, iterations=2, seed=3, stall_mod=2)
    kw = dict(no_prune=True, dump=True)
else:
    regs, p = [I.gen_region(n, 300 + n) for n in (45, 120)], I.Params(ants=64, iterations=2, seed=8)
ids = list(range(len(regs)))
if case == "colony":
    pr = dataclasses.replace(p, ants=32)
    ss = [Scheduler(I.GFX906, device=0) for _ in range(2)]
    keys = []
    for r, s in enumerate(ss):
        s.load(regs, ids)
        keys.append(s.colony_begin(pr, r * 32))
    for pass_ in (1, 2):
        for it in range(pr.iterations):
            for s in ss:
                s.colony_construct(pass_, it)
            m = torch.minimum(keys[0], keys[1])
            for k in keys:
                k.copy_(m)
            for s in ss:
                s.colony_finalize(pass_, it)
    for s in ss:
        s.colony_end()
    got = ss[0].results()
else:
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, ids).run(p, **kw)
    s.run(p, **kw)  # a cached-plan rerun (CUDA graph capture) as well
    got = s.results()
bad = 0
for k, r in enumerate(regs):
    o = O.schedule(r, k, I.GFX906, p)
    ok = got[k]["length"] == o["length"] and got[k]["trace_hash"] == o["trace_hash"] and list(got[k]["order"]) == list(o["order"])
    bad += not ok
print(f"case {case}: {len(regs)} regions, parity {'ok' if not bad else f'{bad} MISMATCH'}")
sys.exit(1 if bad else 0)
