"""Every preemption point (BASELINE north_star: "bit-exact ... for every
preemption point across the 5 configs"): for small instances of C2, C3, C4a
and one C4b level, every warp is preempted at poll visit v in launch 0, for
every v until the kernel runs out of poll visits (and, nested, again at visit
v // 2 of the resume launch), with every register poisoned before the
restore.  Each run must equal the oracle's uninterrupted output bit for bit,
and every saved context must have exactly the bytes of the oracle's plan for
the site the warp reports."""
import numpy as np
import pytest

from oracle import analysis as A
from oracle import interp, ir
from workloads import configs

from gpu_helpers import gpu_run

pytestmark = pytest.mark.gpu


def _cases():
    rp, ci = configs.c4b_graph(1 << 10, 16)
    n = len(rp) - 1
    dist = np.full(n, 0xFFFFFFFF, np.uint32)
    dist[0] = 0
    c4b = dict(ir=configs.c4b_ir(), uniforms={"nf": 1, "lvl1": 1},
               buffers={"rowptr": rp, "colidx": ci, "front": np.zeros(2, np.uint32), "dist": dist,
                        "nextf": np.zeros(n, np.uint32), "nextcnt": np.zeros(1, np.uint32)})
    return {
        "c2": (configs.c2(128, 128, 64, polls="half"), 1, (), 2),
        "c3": (configs.c3(512, 128, 64), 4, (), 0),
        "c3r2": (configs.c3(512, 128, 64, rows_per_iter=2), 4, (), 0),
        "c4a": (configs.c4a(1 << 14, grid=2), 2, (), 0),
        "c4b": (c4b, 2, ("nextf",), 0),     # frontier order is nondeterministic: compared as a multiset
    }


@pytest.mark.parametrize("which", ["c2", "c3", "c3r2", "c4a", "c4b"])
def test_every_poll_visit(which):
    import paper_conf_ipps_jiw21_b200 as cb
    cfg, grid, unordered, mb = _cases()[which]
    op = ir.parse(cfg["ir"])
    an = A.analyze(op, policy="EXPLICIT")
    prog = cb.Program(cfg["ir"], poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_FORCED | cb.DEBUG_POISON,
                      min_blocks_per_sm=mb)
    for k, c in enumerate(an.sites):
        assert prog.plan_text(k) == A.plan_text(op, an.plans[c])
    plan_bytes = [an.plans[c].payload_bytes for c in an.sites]
    live_bytes = [an.live[c].payload_bytes for c in an.sites]
    names = list(op.buffers)
    uni = cfg.get("uniforms", {})
    ref, _ = interp.run(an, grid, cfg["buffers"], uni)
    nw = grid * op.nwarps

    def same(g):
        for nme in names:
            if nme in unordered:
                cnt = int(ref["nextcnt"][0])
                assert np.array_equal(np.sort(g[nme][:cnt]), np.sort(ref[nme][:cnt])), nme
            else:
                assert np.array_equal(g[nme], ref[nme]), nme

    v, total = 0, 0
    while True:
        for nested in (False, True):
            sched = [np.full(nw, v, np.uint32)]
            if nested:
                sched.append(np.full(nw, v // 2, np.uint32))
            g, hdrs, _ = gpu_run(prog, names, grid, cfg["buffers"], uni, schedule=sched)
            same(g)
            pre = 0
            for e, h in enumerate(hdrs):
                for w in range(nw):
                    if h[w, 2] == 1 and h[w, 3] == e + 1:
                        k, live = int(h[w, 0]) & 0x7FFFFFFF, bool(h[w, 0] >> 31)
                        assert int(h[w, 1]) == (live_bytes[k] if live else plan_bytes[k]), (v, e, w, h[w])
                        pre += 1
            if not nested:
                first = pre
            total += pre
        if first == 0:
            break
        v += 1
        assert v < 4096
    print(f"{which}: {v} poll visits swept, {total} warp preemptions checked")
    assert v > 1 and total > 0
