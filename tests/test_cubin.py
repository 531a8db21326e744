"""The compiled sm_100a code, inspected with the CUDA toolkit's own tools
(no GPU needed: NVRTC compiles here).

* `ctxb_program_cubin` exports the cubin; `cuobjdump --dump-resource-usage`
  reads the same register counts as the library's ELF reader (an independent
  read; FULL_HW's bytes, 128 x NUM_REGS per warp, rest on it);
* the save / restore stubs move the context with 128-bit evict-first global
  stores / loads (STG.E.EF.128 / LDG.E.EF.128),
  and the kernels use no local memory (no STL / LDL: no spilled IR
  register), matching the ptxas spill counters in ctxb_program_info_t.
"""
import os
import re
import shutil
import subprocess
import tempfile

import pytest

from workloads import configs

CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
pytestmark = pytest.mark.skipif(not os.path.exists(CUOBJDUMP), reason="cuobjdump not installed")


def _cuobjdump(cubin, *args):
    with tempfile.NamedTemporaryFile(suffix=".cubin", delete=False) as f:
        f.write(cubin)
        path = f.name
    try:
        return subprocess.run([CUOBJDUMP, *args, path], check=True, capture_output=True, text=True).stdout
    finally:
        os.unlink(path)


def cuobjdump_regs(cubin):
    """{function: REG} from `cuobjdump --dump-resource-usage`."""
    out, fn = {}, None
    for line in _cuobjdump(cubin, "--dump-resource-usage").splitlines():
        m = re.match(r"\s*Function (\w+):", line)
        if m:
            fn = m.group(1)
        m = re.search(r"REG:(\d+)\s+STACK:(\d+).*LOCAL:(\d+)", line)
        if m and fn:
            out[fn] = int(m.group(1))
            out[fn + ".stack"] = int(m.group(2))
            out[fn + ".local"] = int(m.group(3))
    return out


def cuobjdump_sass(cubin):
    return _cuobjdump(cubin, "-sass")


def _cb():
    import paper_conf_ipps_jiw21_b200 as cb
    return cb


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4a", "c2_full_hw"])
def test_regcount_matches_cuobjdump(name):
    cb = _cb()
    mode = cb.MODE_FULL_HW if name.endswith("full_hw") else cb.MODE_CTXBACK
    if name == "c1":
        prog = cb.Program(configs.c1()["ir"], debug=cb.DEBUG_FORCED, mode=mode)
    elif name.startswith("c2"):
        prog = cb.Program(configs.c2(256, 256, 64)["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode, min_blocks_per_sm=2)
    elif name == "c3":
        prog = cb.Program(configs.c3(rows_per_iter=2)["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode)
    else:
        prog = cb.Program(configs.c4a(1 << 14, grid=1)["ir"], poll_policy=cb.POLL_EXPLICIT, mode=mode)
    info = prog.info
    cub = prog.cubin()
    assert len(cub) == info["cubin_bytes"] and cub[:4] == b"\x7fELF"
    regs = cuobjdump_regs(cub)
    assert regs["ctxb_run"] == info["num_regs"]
    assert regs["ctxb_resume"] == info["num_regs_resume"]
    # no local memory <=> no spill bytes reported by ptxas
    assert regs["ctxb_run.local"] == 0 and info["spill_stores"] == 0 and info["spill_loads"] == 0
    # the resume kernel: C2's CTXBack resume kernel (128 registers, restore +
    # replay + the peeled copy of the tile loop with its fast / generic
    # iterations) spills to a 16 B stack frame (ptxas: 32 B of spill stores),
    # outside the save / restore stubs; the others do not spill
    assert regs["ctxb_resume.local"] == 0 and regs["ctxb_run.stack"] == 0
    assert info["spill_stores_resume"] <= (32 if name == "c2" else 0)
    assert regs["ctxb_resume.stack"] <= (16 if name == "c2" else 0)
    assert (regs["ctxb_resume.stack"] == 0) == (info["spill_stores_resume"] == 0)


def test_c2_stubs_are_128bit_and_spill_free():
    cb = _cb()
    prog = cb.Program(configs.c2(256, 256, 64)["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
    sass = cuobjdump_sass(prog.cubin())
    ops = re.findall(r"\b(STG|LDG|STL|LDL)(\.[A-Z0-9.]+)?", sass)
    names = ["".join(o) for o in ops]
    run_sass = _cuobjdump(prog.cubin(), "-sass", "-fun", "ctxb_run")
    assert not re.search(r"\b(STL|LDL)\b", run_sass), "local-memory traffic in the normal kernel"
    # the resume kernel's few spill accesses (32 B) are not in
    # the restore stubs: every context load is a 128-bit evict-first LDG
    # C2's plans save 68-70 vector values per warp: the save and restore stubs
    # move them as 128-bit evict-first accesses (one v4 per 4 values)
    n_st = sum(1 for n in names if n.startswith("STG") and n.endswith(".128") and ".EF" in n)
    n_ld = sum(1 for n in names if n.startswith("LDG") and n.endswith(".128") and ".EF" in n)
    assert n_st >= 16 and n_ld >= 16, (n_st, n_ld)


def _resume_sass_order(prog):
    """Offsets of the first EXIT and of the evict-first payload loads in ctxb_resume."""
    sass = _cuobjdump(prog.cubin(), "-sass", "-fun", "ctxb_resume")
    first_exit, ef_loads = None, []
    for line in sass.splitlines():
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(@!?P\d\s+)?(\w+)(\.[A-Z0-9.]+)?", line)
        if not m:
            continue
        off, op, mod = int(m.group(1), 16), m.group(3), m.group(4) or ""
        if op == "EXIT" and first_exit is None:
            first_exit = off
        if op == "LDG" and ".EF" in mod:
            ef_loads.append(off)
    return first_exit, ef_loads


def test_speculative_restore_loads_precede_the_header_test():
    """C3's whole payload (4 loads, <= 16 registers) is loaded
    together with the header, before the header test's EXIT; with
    CTXB_DEBUG_NO_SPEC_RESTORE every payload load follows it."""
    cb = _cb()
    ir_ = configs.c3(**configs.BENCH_C3)["ir"]
    spec = cb.Program(ir_, poll_policy=cb.POLL_EXPLICIT)
    assert spec.source.count("_spec(pay") == 4 and "sdep" in spec.source
    ex, lds = _resume_sass_order(spec)
    assert ex is not None and sum(1 for x in lds if x < ex) == 4, (ex, lds)
    off = cb.Program(ir_, poll_policy=cb.POLL_EXPLICIT, debug=cb.DEBUG_NO_SPEC_RESTORE)
    assert "_spec(pay" not in off.source
    ex, lds = _resume_sass_order(off)
    assert ex is not None and lds and all(x > ex for x in lds), (ex, lds)
    # C2's plans hold 68-70 values: nothing is speculated (register budget)
    c2 = cb.Program(configs.c2(256, 256, 64)["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
    assert "_spec(pay" not in c2.source


def _chunks(cubin, fn):
    """(instructions, FFMA, IMAD) of the straight-line SASS runs between branches of `fn`."""
    out, cur = [], []
    for ln in _cuobjdump(cubin, "-sass", "-fun", fn).splitlines():
        m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
        if not m:
            continue
        op = re.sub(r"^@!?U?P\w+\s+", "", m.group(2)).split()[0]
        cur.append(op)
        if op.startswith("BRA"):
            out.append((len(cur), sum(o.startswith("FFMA") for o in cur), sum(o.startswith("IMAD") for o in cur)))
            cur = []
    return out


def test_c2_resumed_warps_run_the_normal_k_loop():
    """resumed warps run k-iterations as good as the normal
    kernel's -- in the peeled copy of the current tile (the fast path of the
    top-bit test) and in the normal loop they re-enter for the next tile:
    the resume kernel holds at least two 256-FFMA runs with no more address
    IMADs than the normal kernel's (before: 64 more per iteration)."""
    cb = _cb()
    prog = cb.Program(configs.c2()["ir"], poll_policy=cb.POLL_EXPLICIT, min_blocks_per_sm=2)
    cub = prog.cubin()
    run = [c for c in _chunks(cub, "ctxb_run") if c[1] == 256]
    res = [c for c in _chunks(cub, "ctxb_resume") if c[1] == 256]
    best = min(c[2] for c in run)
    fast = [c for c in res if c[2] <= best + 4]
    assert len(fast) >= 2, (run, res)
    src = prog.source
    assert "RT_0:" in src and "copy A of BB" in src and "& 0x80000000u) == 0u" in src
    assert "kernel-invariant registers recomputed" in src
