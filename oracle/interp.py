"""Oracle SIMT interpreter of the IR, with preemption / poison / restore / replay.

Test infrastructure only (see oracle/__init__.py).

Execution model:
  * a thread block has `block` threads = block/32 warps of 32 lanes; vector
    registers hold one u32 per lane, scalar registers one u32 per warp;
    registers start at 0;
  * control flow is warp-uniform; warps are independent (no barriers);
  * integer ops are mod 2^32, shifts by >= 32 give 0 (sar: sign fill);
    f32 ops are IEEE RN without FTZ (oracle.fp32); ffma rounds once;
  * guarded memory ops act only in lanes whose guard is non-zero; a guarded-
    off load yields 0;
  * atomics execute in a defined order: warp, then lane.

Warps that share a program counter are executed together as a "gang" (plain
vectorisation of identical per-warp steps); a gang splits when its warps'
uniform branch conditions differ or some of them are preempted.

Preemption follows the paper's runtime: a warp that reaches a
poll site whose forced target matches is preempted *before* executing the
instruction there.  Its dedicated routine is the site's plan:
at-preempt reverts, then the saved values are stored.  All of its registers
and OSRB slots are then overwritten with a seeded poison, and in the next
launch the resume routine loads the saved values, runs the plan's resume
schedule in value-SSA form, writes LIVE_IN(c) and continues at c (P:313-315,
Figs 2c-6c).  After a resume, until the warp leaves that basic block, a
second preemption uses the LIVE plan of its site (R-16 in DESIGN.md).
"""
from __future__ import annotations

import numpy as np

from . import fp32
from .analysis import MODE_FULL, PRE, Analysis, smem_slice

M32 = 0xFFFFFFFF
NEVER = 0xFFFFFFFF


class OracleError(RuntimeError):
    pass


def _u(x):
    return np.asarray(x, dtype=np.uint32)


def _shl(a, b):
    b = _u(b)
    return np.where(b < 32, a << (b & 31), np.uint32(0)).astype(np.uint32)


def _shr(a, b):
    b = _u(b)
    return np.where(b < 32, a >> (b & 31), np.uint32(0)).astype(np.uint32)


def _sar(a, b):
    b = np.minimum(_u(b), np.uint32(31))
    return (_u(a).view(np.int32) >> b.astype(np.int32)).view(np.uint32)


def _rotl(a, b):
    k = _u(b) & 31
    return np.where(k == 0, a, (a << k) | (a >> ((32 - k) & 31))).astype(np.uint32)


def _rotr(a, b):
    k = _u(b) & 31
    return np.where(k == 0, a, (a >> k) | (a << ((32 - k) & 31))).astype(np.uint32)


def _setp(cmp, typ, a, b):
    if typ == "u":
        x, y = _u(a), _u(b)
    elif typ == "s":
        x, y = _u(a).view(np.int32), _u(b).view(np.int32)
    else:
        x, y = fp32.f(a), fp32.f(b)
    r = {"eq": x == y, "ne": x != y, "lt": x < y, "le": x <= y, "gt": x > y, "ge": x >= y}[cmp]
    return r.astype(np.uint32)


def alu(op, mod, a):
    """Value of an ALU instruction for operand arrays `a` (list)."""
    with np.errstate(over="ignore"):
        if op == "mov":
            return _u(a[0]).copy()
        if op == "not":
            return ~_u(a[0])
        if op == "neg":
            return (np.uint32(0) - _u(a[0])).astype(np.uint32)
        if op == "iadd":
            return (_u(a[0]) + _u(a[1])).astype(np.uint32)
        if op == "isub":
            return (_u(a[0]) - _u(a[1])).astype(np.uint32)
        if op == "imul":
            return (_u(a[0]) * _u(a[1])).astype(np.uint32)
        if op == "imad":
            return (_u(a[0]) * _u(a[1]) + _u(a[2])).astype(np.uint32)
        if op == "and":
            return _u(a[0]) & _u(a[1])
        if op == "or":
            return _u(a[0]) | _u(a[1])
        if op == "xor":
            return _u(a[0]) ^ _u(a[1])
        if op == "shl":
            return _shl(_u(a[0]), a[1])
        if op == "shr":
            return _shr(_u(a[0]), a[1])
        if op == "sar":
            return _sar(a[0], a[1])
        if op == "rotl":
            return _rotl(_u(a[0]), a[1])
        if op == "rotr":
            return _rotr(_u(a[0]), a[1])
        if op == "umin":
            return np.minimum(_u(a[0]), _u(a[1]))
        if op == "umax":
            return np.maximum(_u(a[0]), _u(a[1]))
        if op == "imin":
            return np.minimum(_u(a[0]).view(np.int32), _u(a[1]).view(np.int32)).view(np.uint32)
        if op == "imax":
            return np.maximum(_u(a[0]).view(np.int32), _u(a[1]).view(np.int32)).view(np.uint32)
        if op == "sel":
            return np.where(_u(a[0]) != 0, _u(a[1]), _u(a[2])).astype(np.uint32)
        if op == "setp":
            return _setp(mod[0], mod[1], a[0], a[1])
        if op == "fadd":
            return fp32.fadd(a[0], a[1])
        if op == "fsub":
            return fp32.fsub(a[0], a[1])
        if op == "fmul":
            return fp32.fmul(a[0], a[1])
        if op == "ffma":
            return fp32.ffma(a[0], a[1], a[2])
        if op == "i2f":
            return fp32.i2f(a[0])
        if op == "u2f":
            return fp32.u2f(a[0])
        if op == "f2i":
            return fp32.f2i(a[0])
    raise OracleError(f"not an ALU op: {op}")


def invert(kind, rp, others):
    """R-5 inverses: recover r from r' = op(r, others)."""
    with np.errstate(over="ignore"):
        rp = _u(rp)
        if kind == "sub_d":
            return (rp - _u(others[0])).astype(np.uint32)
        if kind == "add_d":
            return (rp + _u(others[0])).astype(np.uint32)
        if kind == "rsub_d":
            return (_u(others[0]) - rp).astype(np.uint32)
        if kind == "xor_d":
            return rp ^ _u(others[0])
        if kind == "not_d":
            return ~rp
        if kind == "neg_d":
            return (np.uint32(0) - rp).astype(np.uint32)
        if kind == "mulinv":
            inv = pow(int(_u(others[0]).flat[0]), -1, 1 << 32)
            return (rp * np.uint32(inv)).astype(np.uint32)
        if kind == "rotr":
            return _rotr(rp, others[0])
        if kind == "rotl":
            return _rotl(rp, others[0])
    raise OracleError(kind)


class Machine:
    """One kernel execution over a grid (or a subset of its blocks)."""

    def __init__(self, an: Analysis, grid: int, buffers: dict, uniforms: dict | None = None,
                 blocks=None, poison_seed: int = 12345):
        self.an = an
        self.prog = prog = an.prog
        self.grid = grid
        self.blocks = list(range(grid)) if blocks is None else list(blocks)
        nw = prog.nwarps
        self.warp_ids = np.array([b * nw + w for b in self.blocks for w in range(nw)], dtype=np.int64)
        self.nW = len(self.warp_ids)
        self.mem = {k: np.array(v, dtype=np.uint32, copy=True) for k, v in buffers.items()}
        for name in prog.buffers:
            if name not in self.mem:
                raise OracleError(f"missing buffer {name}")
        self.uni = {k: int(v) & M32 for k, v in (uniforms or {}).items()}
        for name in prog.uniforms:
            if name not in self.uni:
                raise OracleError(f"missing uniform {name}")
        self.V = np.zeros((max(prog.nv, 1), self.nW, 32), dtype=np.uint32)
        self.S = np.zeros((max(prog.ns, 1), self.nW), dtype=np.uint32)
        self.slot = {m: np.zeros(self.nW, dtype=np.uint32) for m in an.backups}
        self.backup_set = set(an.backups)
        self.sites = set(an.sites)
        self.bb_starts = {s for (s, _e) in prog.bbs}
        self.label_pc = {lab: prog.bbs[b][0] for lab, b in prog.labels.items()}
        self.rng = np.random.default_rng(poison_seed)
        lane = np.arange(32, dtype=np.uint32)
        wib = (self.warp_ids % nw).astype(np.uint32)
        self.sp_tid = (wib[:, None] * 32 + lane[None, :]).astype(np.uint32)
        self.sp_lane = np.broadcast_to(lane, (self.nW, 32))
        self.sp_ctaid = (self.warp_ids // nw).astype(np.uint32)
        self.sp_warpid = wib
        self.nblk = len(self.blocks)
        self.blk_of = (np.arange(self.nW) // nw).astype(np.int64)     # local block of each warp
        self.smem = np.zeros((self.nblk, max(1, prog.smem)), dtype=np.uint32)   # zero at block start
        self.records = []          # preemption records
        self.status = np.zeros(self.nW, dtype=np.int8)   # 0 run, 1 parked, 2 done
        self.parked = {}           # local warp -> (c, plan, ctx)
        self.resumed_pass = np.zeros(self.nW, dtype=bool)
        # CS-Defer: a preemption decided at site c is carried to the
        # site it defers to; pend[w] = that site + 1 (0 = nothing pending)
        self.pend = np.zeros(self.nW, dtype=np.int64)
        self.defer = dict(an.defer) if an.defer else {c: c for c in an.sites}

    # --- operand access ----------------------------------------------------------
    def _opd(self, o, g):
        k = o.kind
        if k == "v":
            return self.V[o.val][g]
        if k == "s":
            return self.S[o.val][g][:, None]
        if k == "imm":
            return np.uint32(o.val)
        n = o.val
        if n == "tid":
            return self.sp_tid[g]
        if n == "laneid":
            return self.sp_lane[g]
        if n == "ctaid":
            return self.sp_ctaid[g][:, None]
        if n == "warpid":
            return self.sp_warpid[g][:, None]
        if n == "nctaid":
            return np.uint32(self.grid)
        if n == "ntid":
            return np.uint32(self.prog.block)
        if n == "nwarps":
            return np.uint32(self.prog.nwarps)
        return np.uint32(self.uni[n])

    def _full(self, x, n):
        return np.broadcast_to(_u(x), (n, 32))

    def _load(self, ins, g, idx, guard):
        buf = self.mem[ins.buf]
        n = len(g)
        idx = self._full(idx, n)
        act = np.ones((n, 32), dtype=bool) if guard is None else (self._full(guard, n) != 0)
        out = np.zeros((n, 32), dtype=np.uint32)
        ii = idx[act].astype(np.int64)
        if ii.size and (ii.max() >= buf.size):
            raise OracleError(f"out-of-bounds load {ins.buf}[{int(ii.max())}] (size {buf.size})")
        out[act] = buf[ii]
        return out

    def _write(self, reg, g, val):
        n = len(g)
        if reg[0] == "v":
            self.V[int(reg[1:])][g] = self._full(val, n)
        else:
            v = self._full(val, n)
            self.S[int(reg[1:])][g] = v[:, 0]

    # --- one instruction for a gang -----------------------------------------------
    def _exec(self, pc, g):
        ins = self.prog.instrs[pc]
        op = ins.op
        n = len(g)
        if pc in self.backup_set:      # OSRB copy before the overwrite
            r = ins.defreg
            self.slot[pc][g] = self.S[int(r[1:])][g]
        if op in ("bra",):
            return [(g, self.label_pc[ins.target])]
        if op in ("brnz", "brz"):
            cond = self.S[ins.srcs[0].val][g] != 0
            take = cond if op == "brnz" else ~cond
            out = []
            if np.any(take):
                out.append((g[take], self.label_pc[ins.target]))
            if np.any(~take):
                out.append((g[~take], pc + 1))
            out.sort(key=lambda t: int(t[0].min()))
            return out
        if op == "exit":
            self.status[g] = 2
            return []
        if op == "bar":          # reached only when every warp of the block arrived (_run_gangs)
            return [(g, pc + 1)]
        a = [self._opd(o, g) for o in ins.srcs]
        guard = self._opd(ins.guard, g) if ins.guard is not None else None
        if op == "ldg":
            val = self._load(ins, g, self._opd(ins.idx, g), guard)
            self._write(ins.defreg, g, val)
        elif op == "lds":
            idx = self._full(self._opd(ins.idx, g), n)
            act = np.ones((n, 32), dtype=bool) if guard is None else (self._full(guard, n) != 0)
            if np.any(idx[act] >= self.prog.smem):
                raise OracleError("out-of-bounds shared-memory load")
            out = np.zeros((n, 32), dtype=np.uint32)
            rows = np.broadcast_to(self.blk_of[g][:, None], (n, 32))
            out[act] = self.smem[rows[act], idx[act].astype(np.int64)]
            self._write(ins.defreg, g, out)
        elif op == "sts":
            idx = self._full(self._opd(ins.idx, g), n)
            val = self._full(a[0], n)
            act = np.ones((n, 32), dtype=bool) if guard is None else (self._full(guard, n) != 0)
            if np.any(idx[act] >= self.prog.smem):
                raise OracleError("out-of-bounds shared-memory store")
            rows = np.broadcast_to(self.blk_of[g][:, None], (n, 32))
            self.smem[rows[act], idx[act].astype(np.int64)] = val[act]
        elif op == "stg":
            buf = self.mem[ins.buf]
            idx = self._full(self._opd(ins.idx, g), n)
            val = self._full(a[0], n)
            act = np.ones((n, 32), dtype=bool) if guard is None else (self._full(guard, n) != 0)
            ii = idx[act].astype(np.int64)
            if ii.size and ii.max() >= buf.size:
                raise OracleError(f"out-of-bounds store {ins.buf}[{int(ii.max())}]")
            buf[ii] = val[act]
        elif op in ("atom.add", "atom.cas"):
            buf = self.mem[ins.buf]
            idx = self._full(self._opd(ins.idx, g), n)
            act = np.ones((n, 32), dtype=bool) if guard is None else (self._full(guard, n) != 0)
            A0 = self._full(a[0], n)
            A1 = self._full(a[1], n) if op == "atom.cas" else None
            old = np.zeros((n, 32), dtype=np.uint32)
            order = np.argsort(g, kind="stable")
            for wi in order:                 # warp, then lane
                for l in range(32):
                    if not act[wi, l]:
                        continue
                    k = int(idx[wi, l])
                    if k >= buf.size:
                        raise OracleError(f"out-of-bounds atomic {ins.buf}[{k}]")
                    o = buf[k]
                    old[wi, l] = o
                    if op == "atom.add":
                        buf[k] = np.uint32((int(o) + int(A0[wi, l])) & M32)
                    elif o == A0[wi, l]:
                        buf[k] = A1[wi, l]
            if ins.dst is not None:
                self._write(ins.defreg, g, old)
        else:
            self._write(ins.defreg, g, alu(op, ins.mod, a))
        return [(g, pc + 1)]

    # --- preemption -----------------------------------------------------
    def _reg_val(self, r, w):
        if r[0] == "v":
            return self.V[int(r[1:])][w].copy()
        return np.uint32(self.S[int(r[1:])][w])

    def _preempt(self, w, c):
        # R-16: a nested preemption in the resumed BB pass uses the site's LIVE
        # plan (registers dead at c are garbage after the resume).  FULL saves
        # every declared register regardless of liveness (the BASELINE routine
        # "swaps all occupied resources"), so it keeps its plan.
        nested_live = self.resumed_pass[w] and self.an.mode != MODE_FULL
        plan = self.an.live[c] if nested_live else self.an.plans[c]
        tmp = {}
        # at-preempt reverts, decreasing m (Alg.2 MIN_COST at_preempt; Fig 3b, 6b)
        for (v, m, kind, inputs, sups) in plan.preempt_reverts:
            vals = []
            for x, s in zip(inputs, sups):
                if s[0] == "C":
                    vals.append(self._reg_val(x[0], w))
                elif s[0] == "R":
                    vals.append(tmp[x])
                elif s[0] == "B":
                    vals.append(np.uint32(self.slot[s[1]][w]))
                else:
                    raise OracleError("at-preempt revert with a re-executed input")
            others = self._revert_others(m, v[0], vals[1:], w)
            tmp[v] = invert(kind, vals[0], others)
        ctx = {}
        for src, v in plan.saved:
            if src == "C":
                ctx[v] = self._reg_val(v[0], w)
            elif src == "P":
                ctx[v] = tmp[v]
            elif src == "B":
                ctx[v] = np.uint32(self.slot[plan.backup_of[v]][w])
        nbytes = sum(128 if v[0][0] == "v" else 4 for v in ctx)
        assert nbytes == plan.payload_bytes
        lo, hi = smem_slice(self.prog, int(self.warp_ids[w] % self.prog.nwarps))
        b = self.blk_of[w]
        ctx["%smem"] = self.smem[b, lo:hi].copy()
        self.records.append(dict(warp=int(self.warp_ids[w]), site=c, kind=plan.kind,
                                 bytes=plan.payload_bytes + 4 * (hi - lo), p=plan.p, launch=self.cur_launch))
        self.smem[b, lo:hi] = self.rng.integers(0, 1 << 32, hi - lo, dtype=np.uint32)
        # poison every register and slot of the warp (nothing but ctx survives)
        self.V[:, w, :] = self.rng.integers(0, 1 << 32, size=self.V[:, w, :].shape, dtype=np.uint32)
        self.S[:, w] = self.rng.integers(0, 1 << 32, size=self.S[:, w].shape, dtype=np.uint32)
        for m in self.slot:
            self.slot[m][w] = self.rng.integers(0, 1 << 32, dtype=np.uint32)
        self.parked[w] = (c, plan, ctx)
        self.status[w] = 1

    def _revert_others(self, m, x0, vals, w):
        """Operand values of revert m other than the shared register x0:
        register inputs come from `vals` (in order); immediates and specials
        are re-materialised for warp w (they are never saved)."""
        from .analysis import revert_spec
        _kind, others = revert_spec(self.prog.instrs[m], x0)
        out, k = [], 0
        for o in others:
            if o.is_reg:
                out.append(vals[k])
                k += 1
            else:
                x = _u(self._opd(o, np.array([w])))
                out.append(x.reshape(-1)[0] if x.size == 1 else x.reshape(-1, 32)[0])
        return out

    def _resume(self, w):
        """Dedicated resume routine: load, re-execute / revert in schedule
        order (value-SSA), write LIVE_IN(c), continue at c (Figs 2c-6c)."""
        c, plan, ctx = self.parked.pop(w)
        lo, hi = smem_slice(self.prog, int(self.warp_ids[w] % self.prog.nwarps))
        self.smem[self.blk_of[w], lo:hi] = ctx.pop("%smem")
        saved_src = {v: src for src, v in plan.saved}
        res = {}     # ('X', j) -> value ; ('R', v) -> value

        def val(x, s):
            k = s[0]
            if k in ("C", "B"):
                return ctx[x]
            if k == "X":
                return res[("X", s[1])]
            if k == "R":
                if saved_src.get(x) == "P":
                    return ctx[x]
                return res[("R", x)]
            raise OracleError(s)

        ga = np.array([w])
        for ev in plan.schedule:
            if ev[0] == "X":
                j = ev[1]
                ins = self.prog.instrs[j]
                sup = plan.reexec_supply[j]
                regvals = [val(x, s) for x, s in zip(self._opvals(plan, j), sup)]
                res[("X", j)] = self._eval_with(ins, regvals, w)
            else:
                v = ev[1]
                m, kind, inputs, sups = plan.revert_info[v]
                vals = [val(x, s) for x, s in zip(inputs, sups)]
                others = self._revert_others(m, v[0], vals[1:], w)
                res[("R", v)] = invert(kind, vals[0], others)
        for r, s in plan.final.items():
            # s refers to the value (r, rd(r, c))
            if s[0] == "X":
                x = res[("X", s[1])]
            else:
                x = ctx[self._final_value(plan, r)]
            if r[0] == "v":
                self.V[int(r[1:])][w] = np.broadcast_to(_u(x), (32,))
            else:
                self.S[int(r[1:])][w] = _u(x).reshape(-1)[0]
        self.status[w] = 0
        self.resumed_pass[w] = True
        self.pend[w] = 0
        return c

    def _final_value(self, plan, r):
        d = PRE
        for k in range(plan.c - 1, plan.p - 1, -1):
            if self.prog.instrs[k].defreg == r:
                d = k
                break
        return (r, d)

    def _opvals(self, plan, j):
        out = []
        for u in self.prog.instrs[j].uses():
            d = PRE
            for k in range(j - 1, plan.p - 1, -1):
                if self.prog.instrs[k].defreg == u:
                    d = k
                    break
            out.append((u, d))
        return out

    def _eval_with(self, ins, regvals, w):
        """Evaluate a re-executable instruction for warp w with register
        operands taken from `regvals` (uses() order)."""
        k = 0
        ops = []
        g = np.array([w])

        def take(o):
            nonlocal k
            if o.is_reg:
                x = regvals[k]
                k += 1
                return np.broadcast_to(_u(x), (32,))[None, :] if o.kind == "v" else \
                    np.broadcast_to(_u(x).reshape(-1)[:1], (1, 32))
            return self._opd(o, g)
        for o in ins.srcs:
            ops.append(take(o))
        if ins.op == "ldg":
            idx = take(ins.idx)
            guard = take(ins.guard) if ins.guard is not None else None
            out = self._load(ins, g, idx, guard)[0]
        else:
            out = np.broadcast_to(_u(alu(ins.op, ins.mod, ops)), (1, 32))[0]
        if ins.defreg[0] == "s":
            return np.uint32(out[0])
        return out.copy()

    # --- launches ------------------------------------------------------------------
    def _run_gangs(self, gangs, targets, count, landing):
        """Run gangs to completion/preemption.  `landing`: local warp -> site
        it resumed at (no poll there).  A gang reaching `bar` waits until
        every running warp of its block has arrived; a poll site at a barrier
        is decided block-uniformly (any warp's decision preempts the block,
        as __syncthreads_or does)."""
        prog = self.prog
        ni = len(prog.instrs)
        gangs = [(g, pc, False) for g, pc in gangs]
        wait = {}
        while gangs:
            g, pc, released = gangs.pop(0)
            while len(g):
                if pc >= ni:
                    raise OracleError("fell off the end of the kernel")
                ins = prog.instrs[pc]
                if ins.op == "bar" and not released:
                    for w in g:
                        wait.setdefault(int(self.blk_of[w]), []).append(int(w))
                    for b in sorted(set(int(x) for x in self.blk_of[g])):
                        members = np.nonzero((self.blk_of == b) & (self.status == 0))[0]
                        if len(wait.get(b, [])) == len(members):
                            ws = np.array(sorted(wait.pop(b)), dtype=np.int64)
                            gangs.append((ws, pc, True))
                    break
                released = False
                if landing:
                    land = np.array([landing.get(int(w)) == pc for w in g])
                    for w in g:
                        landing.pop(int(w), None)
                else:
                    land = None
                if pc in self.sites:
                    pw = g if land is None else g[~land]
                    if len(pw):
                        hit = count[pw] == targets[pw]
                        count[pw] += 1
                        if ins.op == "bar":
                            # block-uniform: OR of the warps' decisions per block
                            bl = self.blk_of[pw]
                            anyhit = np.array([hit[bl == b].any() for b in bl])
                            hit = anyhit
                        pend = self.pend[pw]
                        save = (pend == pc + 1)                      # a deferred preemption lands here
                        start = (pend == 0) & hit
                        d = self.defer.get(pc, pc)
                        if d != pc:
                            self.pend[pw[start]] = d + 1             # continue to the deferral target
                        else:
                            save = save | start
                        self.pend[pw[save]] = 0
                        if np.any(save):
                            for w in pw[save]:
                                self._preempt(int(w), pc)
                            g = g[~np.isin(g, pw[save])]
                            if not len(g):
                                break
                outs = self._exec(pc, g)
                if not outs:
                    break
                for gg, npc in outs:
                    if npc in self.bb_starts:
                        self.resumed_pass[gg] = False
                if len(outs) == 1:
                    g, pc = outs[0]
                else:
                    gangs[0:0] = [(x, y, False) for x, y in outs[1:]]
                    g, pc = outs[0]
        if wait:
            raise OracleError("warps left waiting at a barrier (non-uniform barrier)")

    def run(self, schedule=()):
        """Run launch 0 and as many resume launches as needed.

        schedule[k][w] = target poll-visit index (0-based, counted from the
        warp's (re)start in launch k) at which warp w (position in the
        block-ordered list of simulated warps) is preempted; NEVER/absent =
        not preempted.  Returns the final buffers."""
        launch = 0
        while True:
            self.cur_launch = launch
            t = np.full(self.nW, NEVER, dtype=np.int64)
            if launch < len(schedule) and schedule[launch] is not None:
                s = np.asarray(schedule[launch], dtype=np.int64)
                t[:len(s)] = s
            count = np.zeros(self.nW, dtype=np.int64)
            landing = {}
            if launch == 0:
                gangs = [(np.arange(self.nW), 0)]
            else:
                bysite = {}
                for w in sorted(self.parked):
                    c = self._resume(w)
                    landing[w] = c
                    bysite.setdefault(c, []).append(w)
                gangs = [(np.array(ws), c) for c, ws in sorted(bysite.items())]
            self._run_gangs(gangs, t, count, landing)
            launch += 1
            if not self.parked:
                break
            if launch > 10000:
                raise OracleError("too many launches")
        self.launches = launch
        return self.mem


def run(an: Analysis, grid: int, buffers: dict, uniforms=None, schedule=(), blocks=None,
        poison_seed=12345):
    m = Machine(an, grid, buffers, uniforms, blocks, poison_seed)
    mem = m.run(schedule)
    return mem, m.records
