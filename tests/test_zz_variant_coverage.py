"""Every construct-kernel variant a benchmark line launches is covered by an
every-ant (dump-mode) parity test.

The variants of a run are planned on the host (aco_last_variants after a
sizing call: nothing runs); the dump-parity tests of this session record the
variants they exercised in tests.test_gpu_parity.DUMP_VARIANTS.  This file is
named to run last; run on its own (no parity tests before it) it skips.
"""
import os
import sys

import pytest

from tests.test_gpu_parity import DUMP_VARIANTS

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# the benchmark lines of bench.py / tools/bench_matrix.sh
BENCH_LINES = [
    ["--workload", "c1"], ["--workload", "c2"], ["--workload", "c3"], ["--workload", "c4"],
    ["--workload", "c5"], ["--workload", "c3", "--machine", "dual"], ["--workload", "c3", "--passes", "4"],
    ["--workload", "c3", "--policy", "paper"], ["--workload", "c3", "--heur-mix", "1"],
    ["--workload", "c3", "--stall-num", "2"], ["--workload", "c3", "--rl-limit", "1"],
]


def decode(code):
    if code & (1 << 13):
        return "fused"
    lanes = [1, 2, 4, 8][(code >> 6) & 3]
    if code & (1 << 9):
        lanes = 32 if code & (1 << 10) else 16
    f = [f"pass{2 if code & 256 else 1}", f"lanes{lanes}"]
    for bit, name in ((0, "wide"), (1, "gstate"), (2, "nc4"), (3, "t32"), (4, "tau_smem"), (5, "mask"),
                      (11, "img_l1"), (12, "lean")):
        if code & (1 << bit):
            f.append(name)
    return "+".join(f)


_LOADED = {}


def bench_variants(argv):
    """Variants the bench line would launch: its batches loaded once per
    (workload, machine), planned with the line's parameters."""
    import bench
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
    args = bench.parse(argv)
    batches, _, _ = bench.workload(args, 0, 1) if (args.workload, args.machine) not in _LOADED else (None, 0, 0)
    if (args.workload, args.machine) not in _LOADED:
        scheds = []
        for b in batches:
            s = Scheduler(bench.machine_of(args), device=0)
            s.load(b.regs, b.ids)
            scheds.append(s)
        _LOADED[(args.workload, args.machine)] = scheds
    scheds = _LOADED[(args.workload, args.machine)]
    params = [b.p for b in bench.workload(args, 0, 1, gen=False)[0]]
    codes = set()
    for s, p in zip(scheds, params):
        codes |= set(s.plan_variants(p))
    return codes


def test_bench_variants_have_every_ant_parity():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    if len(DUMP_VARIANTS) < 4:
        pytest.skip("run with the whole GPU suite (the dump-parity tests record their variants)")
    if ROOT not in sys.path:
        sys.path.insert(0, ROOT)
    missing = {}
    for argv in BENCH_LINES:
        for c in bench_variants(argv) - DUMP_VARIANTS:
            missing.setdefault(decode(c), []).append(" ".join(argv))
    print("dump-parity variants:", sorted(decode(c) for c in DUMP_VARIANTS))
    assert not missing, f"bench variants without every-ant parity: {missing}"
