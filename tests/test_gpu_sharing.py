"""GPU parity of P:317 routine sharing (NEXT N3): sites that enter their
flashback-point's shared preemption routine at an offset (reverts in place)
save exactly their own plan's values.  Forced preemption at every site and at
random per-warp sites, nested, with poisoned resumes; outputs bit-exact with
the oracle and per-warp header bytes equal to the oracle's."""
import json
import os

import numpy as np
import pytest

from oracle import ir
from workloads.randprog import random_buffers, random_program

from test_gpu_parity import check
from test_routine_sharing import FP_SHARED

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_n3_fixture_every_site():
    g = json.load(open(os.path.join(GOLD, "n3.json")))
    op = ir.parse(g["ir"])
    r = np.random.default_rng(3)
    bufs = {b: (r.integers(0, 1 << 32, 64, dtype=np.uint64).astype(np.uint32) if k == "ro" else np.zeros(64, np.uint32))
            for b, k in op.buffers.items()}
    n = len(op.instrs)
    scheds = [[[k]] for k in range(n)] + [[[k], [j]] for k in range(3, 9) for j in range(0, 4)]
    prog, _an = check(g["ir"], 1, bufs, scheds)
    assert prog.info["n_fp_shared"] == len(g["group_sites"])


@pytest.mark.parametrize("seed,loop", FP_SHARED)
def test_random_programs_with_shared_routines(seed, loop):
    txt, size = random_program(seed, loop=loop, n_body=12, fp=False)
    op = ir.parse(txt)
    grid = 3
    nout = op.nv - 1 + op.ns - (1 if loop else 0)
    bufs = random_buffers(seed, op.block, grid, size, nout)
    r = np.random.default_rng(seed)
    nw = grid * op.nwarps
    scheds = [[r.integers(0, 80, nw).astype(np.uint32), r.integers(0, 20, nw).astype(np.uint32)] for _ in range(6)]
    prog, _an = check(txt, grid, bufs, scheds)
    assert prog.info["n_fp_shared"] >= 2
