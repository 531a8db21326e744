"""The two independent IR parsers (oracle/ir.py, csrc/ir.cpp) accept and
reject the same texts: seeded token-level mutations of valid kernels."""
import numpy as np
import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import ir
from workloads import configs
from workloads.randprog import random_program

TOKENS = ["v0", "v99", "s0", "s9", "%tid", "%bogus", "0x10", "-5", "0f3F800000", "4294967296", "-2147483649",
          "iadd", "ldg", "stg", "bar", "lds", "sts", "exit", "bra", "poll", "@v1", "in0[v0]", "nosuch[v0]",
          ",", "", "L0:", ".smem 16", ".vregs 2", "atom.add", "_", "rotl", "setp.lt.u", "setp.xx.u"]


def mutate(text, rng):
    lines = text.splitlines()
    k = int(rng.integers(len(lines)))
    toks = lines[k].replace(",", " , ").split()
    op = int(rng.integers(4))
    if op == 0 and toks:
        toks[int(rng.integers(len(toks)))] = TOKENS[int(rng.integers(len(TOKENS)))]
    elif op == 1:
        toks.insert(int(rng.integers(len(toks) + 1)), TOKENS[int(rng.integers(len(TOKENS)))])
    elif op == 2 and toks:
        del toks[int(rng.integers(len(toks)))]
    else:
        lines.insert(k, "  " + " ".join(TOKENS[int(rng.integers(len(TOKENS)))] for _ in range(3)))
        return "\n".join(lines) + "\n"
    lines[k] = "  " + " ".join(toks).replace(" , ", ", ")
    return "\n".join(lines) + "\n"


def accepts_py(t):
    try:
        ir.parse(t)
        return True
    except ir.IRError:
        return False


def accepts_cpp(t):
    try:
        cb.Program(t, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_COMPILE)
        return True
    except cb.CtxbError as e:
        assert e.code == -2, str(e)
        return False


@pytest.mark.parametrize("seed", range(4))
def test_parsers_agree_on_mutations(seed):
    rng = np.random.default_rng(seed)
    bases = [configs.C1_IR, configs.c3_ir(512, 128, 64), configs.c4b_ir(), random_program(seed, loop=True)[0]]
    n_acc = n_rej = 0
    for base in bases:
        for _ in range(60):
            t = mutate(base, rng)
            a, b = accepts_py(t), accepts_cpp(t)
            assert a == b, t
            n_acc += a
            n_rej += not a
    assert n_acc > 0 and n_rej > 0
