"""P:317 routine sharing (NEXT N3): one preemption routine per flashback-point
whose reverting part nests, entered at an offset per site.

tests/golden/n3.json fixes by hand (from P:317's rule) which sites share the
routine and at which offsets; the generated code must realise exactly that,
with the reverts applied in place in decreasing instruction order.  Sharing
changes only the code, never the plans (plan text == oracle)."""
import json
import os
import re

import pytest

import paper_conf_ipps_jiw21_b200 as cb
from oracle import analysis as A
from oracle import ir
from workloads import configs
from workloads.randprog import random_program

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ENTRY = re.compile(r"SAVE_(\d+): sid = \d+u; t_seen_e = [^;]*; (?:__syncwarp\(\); )?goto SAVE_F(\d+)_E(\d+);")

# integer-only random programs (randprog seeds, loop) in which P:317 sharing applies
FP_SHARED = [(24, True), (38, True), (43, False), (74, False), (99, False), (156, True), (178, False), (237, False)]


def entries(src):
    return {int(k): (int(g), int(e)) for k, g, e in ENTRY.findall(src)}


def test_n3_fixture_by_hand():
    g = json.load(open(os.path.join(GOLD, "n3.json")))
    op = ir.parse(g["ir"])
    an = A.analyze(op)
    prog = cb.Program(g["ir"], debug=cb.DEBUG_NO_COMPILE)
    for c in g["group_sites"]:
        assert an.plans[c].p == g["p"] and an.plans[c].payload_bytes == g["bytes"]
        si = prog.site_info(an.sites.index(c))
        assert si["p"] == g["p"] and si["payload_bytes_per_warp"] == g["bytes"]
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    src = prog.source
    got = entries(src)
    want = {an.sites.index(int(c)): e for c, e in g["entry"].items()}
    assert {k: e for k, (grp, e) in got.items()} == want
    assert len({grp for grp, _ in got.values()}) == 1
    # the master routine: in-place reverts in decreasing m, one entry label before each
    body = src[src.index("SAVE_F0_E0:"):]
    ms = [int(m) for m in re.findall(r"// revert I(\d+) in place", body.split("SAVE_F0_E%d:" % len(g["reverts_in_master_order"]))[0])]
    assert ms == g["reverts_in_master_order"]
    info = prog.info
    assert info["n_fp_shared"] == len(g["group_sites"])
    base = cb.Program(g["ir"], debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_FP_SHARE).info
    assert info["n_save_stubs"] < base["n_save_stubs"]


@pytest.mark.parametrize("seed,loop", FP_SHARED)
def test_random_programs_share_and_keep_plans(seed, loop):
    txt, _ = random_program(seed, loop=loop, n_body=12, fp=False)
    op = ir.parse(txt)
    an = A.analyze(op)
    prog = cb.Program(txt, debug=cb.DEBUG_NO_COMPILE)
    assert prog.info["n_fp_shared"] >= 2
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    base = cb.Program(txt, debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_FP_SHARE).info
    assert prog.info["n_save_stubs"] < base["n_save_stubs"]
    # every member shares its master's flashback-point and saved values
    groups = {}
    for k, (grp, _e) in entries(prog.source).items():
        groups.setdefault(grp, []).append(k)
    for ks in groups.values():
        pls = [an.plans[an.sites[k]] for k in ks]
        assert len({pl.p for pl in pls}) == 1
        assert len({tuple(v for _s, v in pl.saved) for pl in pls}) == 1


def test_configs_unchanged():
    """On the bench configs the rule never applies beyond exact sharing (C1's
    plans have no at-preempt reverts; C2's sites with one flashback-point
    save different values): routine counts are those of exact sharing."""
    for txt, pol, mb in ((configs.c1()["ir"], cb.POLL_EVERY_INSTR, 0),
                         (configs.c2(256, 256, 64, polls="half")["ir"], cb.POLL_EXPLICIT, 2)):
        a = cb.Program(txt, poll_policy=pol, min_blocks_per_sm=mb, debug=cb.DEBUG_NO_COMPILE).info
        b = cb.Program(txt, poll_policy=pol, min_blocks_per_sm=mb,
                       debug=cb.DEBUG_NO_COMPILE | cb.DEBUG_NO_FP_SHARE).info
        assert a["n_save_stubs"] == b["n_save_stubs"] and a["n_fp_shared"] == 0
