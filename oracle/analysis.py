"""Oracle flashback analysis: liveness, windows, the CTXB-R1 sweep, plans.

Test infrastructure only (see oracle/__init__.py).  Deliberately naive: every
(site c, candidate p) pair is recomputed from scratch (R-9 forbids reusing
marks across p), with Python sets and dicts, in the order the paper and
DESIGN.md "Normative reading CTXB-R1" state.

Paper passages followed (PAPER.md line numbers, `P:n`):
  * register context of an instruction = its live-in registers
  * preemption signal handled *before* I_cur; window [I_prec, I_cur) P:74 (R-1)
  * relaxed condition: every live-out result in the window restorable by
    re-execution or save/reload                                   P:90-116, Alg.1 P:120-143 (R-2)
  * instruction reverting, Alg. 2 (availability: not overwritten /
    recoverable by revert / re-executable; at_resume forcing;
    MIN_COST position)                                            P:154-231 (R-5, R-6)
  * OSRB: back up scalars that give better flashback-points       P:257-269 (R-7)
  * combined fixpoint of the three methods                        P:271-303 (R-9)
  * windows limited to the basic block and idempotent region      P:305 (R-3)
  * per instruction, pick the least-latency flashback-point       P:313, P:337 (R-10)
  * context = saved values incl. results restored by save/reload  P:343 (R-8)

Value notation: (r, d) is the value of register r produced by instruction d
(a global instruction index inside the window) or d = PRE (None): r's value
on entry to the window.
"""
from __future__ import annotations

import bisect
from dataclasses import dataclass, field

from .ir import Program

PRE = None

# --- instruction classes (DESIGN.md "IR v1" table; R-4, R-5) -----------------

ALU_OPS = {"mov", "not", "neg", "i2f", "u2f", "f2i", "iadd", "isub", "imul", "and", "or",
           "xor", "shl", "shr", "sar", "rotl", "rotr", "umin", "umax", "imin", "imax",
           "fadd", "fsub", "fmul", "ffma", "imad", "sel", "setp"}

FLAG_RELAXED = 1
FLAG_REVERT = 2
FLAG_OSRB = 4
FLAGS_ALL = 7
FLAG_DEFER = 8            # CS-Defer on top of the mode's own plans
FLAG_PRUNE = 16           # demand-driven restore (NEXT N4): restore only what LIVE_IN(c) needs
FLAG_RANK_RESUME = 32     # combined preempt + resume ranking of flashback-points (NEXT N4)
FLAG_EXACT = 64           # exact minimum-bytes saved set per window (NEXT N4, oracle/exact.py)

DEFER_INSTR_BYTES = 8     # latency-estimate weight of one deferred instruction, in context bytes
RESUME_LEVEL_BYTES = 512  # FLAG_RANK_RESUME: one dependent memory round trip, in context bytes

MODE_CTXBACK = 0
MODE_LIVE = 1
MODE_FULL = 2

VEC_BYTES = 128   # one 32-bit register x 32 lanes per warp  (R-8)
SCA_BYTES = 4     # one uniform 32-bit register per warp       (R-8)


def reexec_op_kind(prog: Program, ins) -> bool:
    """R-4: ALU ops and loads from read-only buffers can be re-executed.
    Loads from rw buffers or shared memory (written by other warps), atomics,
    stores, barriers and control flow cannot."""
    if ins.op in ALU_OPS:
        return True
    if ins.op == "ldg":
        return prog.buffers[ins.buf] == "ro"
    return False


def _inv_odd(a: int) -> int:
    """Multiplicative inverse of an odd a modulo 2^32 (closed form via pow)."""
    return pow(a, -1, 1 << 32)


def revert_spec(ins, r):
    """R-5: is `ins` of the form r' = op(r, {R}) with a bit-exact inverse?

    Returns None (irreversible) or a pair (kind, others): `others` are the
    operands of ins other than the shared register r (registers, immediates or
    specials), and `kind` names the inverse:
      'sub_d'  : r = r' - x          (iadd r, r, x | iadd r, x, r)
      'add_d'  : r = r' + x          (isub r, r, x)
      'rsub_d' : r = x - r'          (isub r, x, r)
      'xor_d'  : r = r' ^ x          (xor  r, r, x | xor r, x, r)
      'not_d'  : r = ~r'             (not  r, r)
      'neg_d'  : r = -r'             (neg  r, r)
      'mulinv' : r = r' * inv(k)     (imul r, r, k | imul r, k, r; k odd immediate)
      'rotr'   : r = rotr(r', k)     (rotl r, r, k; k immediate)
      'rotl'   : r = rotl(r', k)     (rotr r, r, k; k immediate)
    SHL and every f32 op are irreversible (bits lost / rounding).
    """
    if ins.dst is None or ins.defreg != r or ins.op == "lds":
        return None
    s = ins.srcs
    regs = [o.reg for o in s if o.is_reg]
    if regs.count(r) != 1:
        return None
    if ins.guard is not None or ins.idx is not None:
        return None
    op = ins.op
    if op in ("not", "neg"):
        return (op + "_d", [])
    if len(s) != 2:
        return None
    a, b = s
    if op == "iadd":
        return ("sub_d", [b if a.reg == r else a])
    if op == "isub":
        return ("add_d", [b]) if a.reg == r else ("rsub_d", [a])
    if op == "xor":
        return ("xor_d", [b if a.reg == r else a])
    if op == "imul":
        other = b if a.reg == r else a
        if other.kind == "imm" and other.val % 2 == 1:
            return ("mulinv", [other])
        return None
    if op in ("rotl", "rotr") and a.reg == r and b.kind == "imm":
        return ("rotr" if op == "rotl" else "rotl", [b])
    return None


# --- liveness ------------------------------------------------------------

@dataclass
class Liveness:
    live_in: list    # per global instruction: frozenset of registers live before it
    live_out: list   # per global instruction: frozenset live after it


def liveness(prog: Program) -> Liveness:
    """Standard backward iterative dataflow over the CFG (textbook liveness).
    IR registers are zero-initialised at kernel entry, so a register live at
    entry is simply a read of that initial value."""
    nb = len(prog.bbs)
    use_b = [set() for _ in range(nb)]
    def_b = [set() for _ in range(nb)]
    for b, (s, e) in enumerate(prog.bbs):
        for i in range(s, e):
            ins = prog.instrs[i]
            for r in ins.uses():
                if r not in def_b[b]:
                    use_b[b].add(r)
            if ins.defreg:
                def_b[b].add(ins.defreg)
    lin = [set() for _ in range(nb)]
    lout = [set() for _ in range(nb)]
    changed = True
    while changed:
        changed = False
        for b in reversed(range(nb)):
            o = set()
            for sb in prog.bb_succ[b]:
                o |= lin[sb]
            i_ = use_b[b] | (o - def_b[b])
            if o != lout[b] or i_ != lin[b]:
                lout[b], lin[b] = o, i_
                changed = True
    n = len(prog.instrs)
    live_in = [None] * n
    live_out = [None] * n
    for b, (s, e) in enumerate(prog.bbs):
        cur = set(lout[b])
        for i in reversed(range(s, e)):
            ins = prog.instrs[i]
            live_out[i] = frozenset(cur)
            if ins.defreg:
                cur.discard(ins.defreg)
            cur |= set(ins.uses())
            live_in[i] = frozenset(cur)
    return Liveness(live_in, live_out)


# --- windows: basic block + idempotent region heads (R-3) -----------------

def region_heads(prog: Program) -> list:
    """h(c) for every site position c (a global instruction index; the site is
    *before* instruction c).  h(c) = max(BB start, region start), where a new
    idempotent region starts after every atomic and every barrier, and *at* a
    store to buffer b (or shared memory) if b was loaded earlier in the
    current region (memory WAR clobber)."""
    n = len(prog.instrs)
    heads = [0] * n
    for (s, e) in prog.bbs:
        head = s
        loaded = set()
        for c in range(s, e):
            heads[c] = head
            ins = prog.instrs[c]
            # boundaries triggered by instruction c apply to sites > c
            if ins.op in ("atom.add", "atom.cas", "bar"):
                head = c + 1
                loaded = set()
            elif ins.op in ("stg", "sts") and ins.buf in loaded:
                head = c
                loaded = set()
            elif ins.op in ("ldg", "lds"):
                loaded.add(ins.buf)
    return heads


def sites_for_policy(prog: Program, policy: str, every: int = 8) -> list:
    """Poll-site positions (global instruction indices, site before the instr).
    EVERY_INSTR: before every instruction.  EXPLICIT: the IR's `poll` markers.
    EVERY_N: before BB-local index i for i % N == 0 and i > 0, plus before the
    terminator of every BB that ends in a backward branch.
    Kernels with barriers (N2): preemption is block-uniform and fused with a
    barrier, so the sites are the `bar` instructions (EXPLICIT: the polls, all
    of which precede a `bar`)."""
    if prog.has_barriers and policy != "EXPLICIT":
        return [i for i, ins in enumerate(prog.instrs) if ins.op == "bar"]
    if policy == "EVERY_INSTR":
        return list(range(len(prog.instrs)))
    if policy == "EXPLICIT":
        return sorted(set(prog.explicit_sites))
    if policy == "EVERY_N":
        out = set()
        for b, (s, e) in enumerate(prog.bbs):
            for i in range(s + every, e, every):
                out.add(i)
            last = prog.instrs[e - 1]
            if last.op in ("bra", "brnz", "brz") and prog.labels[last.target] <= b:
                out.add(e - 1)
        return sorted(out)
    raise ValueError(policy)


# --- plans -----------------------------------------------------------------------

@dataclass
class Plan:
    """A flashback plan for site c with flashback-point p."""
    c: int
    p: int
    kind: str                      # 'ctxback' | 'live' | 'full' | 'basic'
    saved: list                    # ordered saved values: (src, (r, d)); src in C/P/B
    preempt_reverts: list          # [(value, m, kind, input_values, input_supplies)] in decreasing m
    schedule: list                 # resume events: ('X', j) | ('R', value)
    reexec_supply: dict            # j -> list of supplies per operand register (in uses() order)
    revert_info: dict              # value -> (m, kind, inputs, supplies)
    final: dict                    # r -> supply of (r, rd(r, c)) for r in LIVE_IN(c)
    payload_bytes: int
    n_vec: int
    n_sca: int
    n_revert_pre: int
    n_revert_res: int
    n_reexec: int
    backup_of: dict = field(default_factory=dict)   # BACKUP value -> OSRB instruction m

    def cost(self):
        """R-10: (bytes, #revert-at-preempt, #resume ops, -p) lexicographic."""
        return (self.payload_bytes, self.n_revert_pre, self.n_reexec + self.n_revert_res, -self.p)


def _bytes_of(prog, vals):
    return sum(VEC_BYTES if prog.is_vector(r) else SCA_BYTES for (r, _d) in vals)


class _Window:
    """State of one (c, p) evaluation: the CTXB-R1 sweep."""

    def __init__(self, prog, lv, p, c, backups, flags):
        self.prog, self.lv, self.p, self.c = prog, lv, p, c
        self.flags = flags
        self.W = list(range(p, c))
        self.valid = {}          # value -> derivation: ('C',) | ('B', m) | ('X', j) | ('R', m)
        self.rev = {}            # value -> (m, kind, inputs, supplies)
        self.reexec = {}         # j -> supplies (per operand register, uses() order)
        self.events = []         # establishment order
        ins = prog.instrs
        # sorted def positions of every register inside the window [p, c)
        self.defs = {}
        for k in range(p, c):
            if ins[k].defreg is not None:
                self.defs.setdefault(ins[k].defreg, []).append(k)
        for r in prog.all_regs():
            self.valid[(r, self.rd(r, c))] = ("C",)
        for m in sorted(backups):
            if p <= m < c:
                s = ins[m].defreg
                v = (s, self.rd(s, m))
                if v not in self.valid:
                    self.valid[v] = ("B", m)

    # rd(r, t): last def of r in [p, t), else PRE
    def rd(self, r, t):
        d = self.defs.get(r)
        if not d:
            return PRE
        i = bisect.bisect_left(d, t)
        return d[i - 1] if i > 0 else PRE

    # nd(r, t): first def of r in [t, c), else None
    def nd(self, r, t):
        d = self.defs.get(r)
        if not d:
            return None
        i = bisect.bisect_left(d, t)
        return d[i] if i < len(d) else None

    def is_current(self, v):
        r, d = v
        return self.nd(r, self.p if d is PRE else d + 1) is None

    def opvals(self, j):
        return [(u, self.rd(u, j)) for u in self.prog.instrs[j].uses()]

    def liveout_def(self, j):
        r = self.prog.instrs[j].defreg
        return r is not None and r in self.lv.live_out[j]

    def reexec_kind(self, j):
        # R-2: dead-result instructions and stores are never re-executed.
        return self.liveout_def(j) and reexec_op_kind(self.prog, self.prog.instrs[j])

    def supply_of(self, v):
        """Snapshot supply (R-9): REEXEC(k) if the producer k is already
        re-executable, else the value's recorded derivation."""
        r, d = v
        if d is not PRE and d in self.reexec:
            return ("X", d)
        return self.valid[v]

    def try_revert(self, v):
        """Alg. 2: recover v = (r, d) by reverting m = nd(r, d+1).
        Inputs: (r, m) and each other register operand value of m at m; each
        is CURRENT (preferred) | already valid | recursively reverted."""
        if not (self.flags & FLAG_REVERT):
            return False
        r, d = v
        m = self.nd(r, self.p if d is PRE else d + 1)
        if m is None:
            return False
        spec = revert_spec(self.prog.instrs[m], r)
        if spec is None:
            return False
        kind, others = spec
        inputs = [(r, m)] + [(o.reg, self.rd(o.reg, m)) for o in others if o.is_reg]
        supplies = []
        for x in inputs:
            if self.is_current(x):
                supplies.append(("C",))
            elif x in self.valid:
                supplies.append(self.supply_of(x))
            elif self.try_revert(x):
                supplies.append(self.valid[x])
            else:
                return False
        self.valid[v] = ("R", m)
        self.rev[v] = (m, kind, inputs, supplies)
        self.events.append(("R", v))
        return True

    def sweep(self):
        changed = True
        while changed:
            changed = False
            for j in self.W:
                if j in self.reexec or not self.reexec_kind(j):
                    continue
                ov = self.opvals(j)
                for x in ov:
                    if x not in self.valid and self.try_revert(x):
                        changed = True
                if all(x in self.valid for x in ov):
                    self.reexec[j] = [self.supply_of(x) for x in ov]
                    self.events.append(("X", j))
                    v = (self.prog.instrs[j].defreg, j)
                    if v not in self.valid:
                        self.valid[v] = ("X", j)
                    changed = True
            for j in self.W:
                if self.liveout_def(j):
                    v = (self.prog.instrs[j].defreg, j)
                    if v not in self.valid and self.try_revert(v):
                        changed = True

    def feasible(self):
        return all((self.prog.instrs[j].defreg, j) in self.valid
                   for j in self.W if self.liveout_def(j))

    # --- context accounting (R-6, R-8) ---

    def demands(self):
        """Resume-time demands: (value, supply) pairs.  R-2 (literal): every
        re-executable instruction's operands and every live-out result of the
        window.  FLAG_PRUNE: only the final value of each register live-in at
        I_cur; re-executions are then demanded transitively (compute_S)."""
        if self.flags & FLAG_PRUNE:
            out = []
            for r in sorted(self.lv.live_in[self.c]):
                d = self.rd(r, self.c)
                out.append(((r, d), self.supply_of((r, d)) if d is not PRE else ("C",)))
            return out
        out = []
        for j in self.W:
            if j in self.reexec:
                out.extend(zip(self.opvals(j), self.reexec[j]))
        for j in self.W:
            if self.liveout_def(j) and j not in self.reexec:
                v = (self.prog.instrs[j].defreg, j)
                out.append((v, self.valid[v]))
        for r in sorted(self.lv.live_in[self.c]):
            if self.rd(r, self.c) is PRE:
                out.append(((r, PRE), ("C",)))
        return out

    def compute_S(self, pos):
        """Saved set S, reverts run at resume, reverts run at preempt (and,
        with FLAG_PRUNE, the re-executions the demands reach)."""
        S = {}
        used_res, used_pre = set(), set()
        used_x = set()
        prune = bool(self.flags & FLAG_PRUNE)

        def pre_closure(v):
            if v in used_pre:
                return
            used_pre.add(v)
            _m, _k, ins_, sups = self.rev[v]
            for x, s in zip(ins_, sups):
                if s[0] == "R":
                    pre_closure(x)

        def demand(v, s):
            k = s[0]
            if k == "C":
                S.setdefault(v, "C")
            elif k == "B":
                S.setdefault(v, "B")
            elif k == "X":
                j = s[1]
                if prune and j not in used_x:
                    used_x.add(j)
                    for x, sx in zip(self.opvals(j), self.reexec[j]):
                        demand(x, sx)
            elif k == "R":
                if pos.get(v, "R") == "P":
                    S.setdefault(v, "P")
                    pre_closure(v)
                else:
                    if v in used_res:
                        return
                    used_res.add(v)
                    _m, _k, ins_, sups = self.rev[v]
                    for x, sx in zip(ins_, sups):
                        demand(x, sx)
        for v, s in self.demands():
            demand(v, s)
        self._used_x = used_x if prune else set(self.reexec)
        return S, used_res, used_pre

    def plan(self, kind="ctxback"):
        prog = self.prog
        pos = {v: "R" for v in self.rev}
        _S0, used0, _ = self.compute_S(pos)
        for v in sorted(used0, key=lambda x: -self.rev[x][0]):
            m, _k, ins_, sups = self.rev[v]
            forced = any(s[0] == "X" or (s[0] == "R" and pos[x] == "R") for x, s in zip(ins_, sups))
            if forced:
                continue
            pos[v] = "P"
            bP = _bytes_of(prog, self.compute_S(pos)[0])
            pos[v] = "R"
            bR = _bytes_of(prog, self.compute_S(pos)[0])
            if bP < bR:
                pos[v] = "P"
        S, used_res, used_pre = self.compute_S(pos)
        used_x = self._used_x
        saved = sorted(((src, v) for v, src in S.items()), key=_saved_key)
        pre_list = sorted(used_pre, key=lambda x: -self.rev[x][0])
        preempt_reverts = [(v,) + tuple(self.rev[v]) for v in pre_list]
        schedule = [e for e in self.events
                    if (e[0] == "X" and e[1] in used_x) or (e[0] == "R" and e[1] in used_res)]
        final = {}
        for r in sorted(self.lv.live_in[self.c]):
            d = self.rd(r, self.c)
            final[r] = self.supply_of((r, d)) if d is not PRE else ("C",)
        nb = _bytes_of(prog, S)
        nv = sum(1 for v in S if prog.is_vector(v[0]))
        bkp = {v: d[1] for v, d in self.valid.items() if d[0] == "B"}
        return Plan(self.c, self.p, kind, saved, preempt_reverts, schedule,
                    {j: self.reexec[j] for j in used_x}, dict(self.rev), final, nb, nv, len(S) - nv,
                    len(used_pre), len(used_res), len(used_x), bkp)


def _saved_key(item):
    src, (r, d) = item
    return (0 if r[0] == "v" else 1, int(r[1:]), -1 if d is PRE else d, src)


def plan_window(prog, lv, p, c, backups=(), flags=FLAGS_ALL):
    """CTXB-R1 plan for flashback-point p of site c, or None if p is not a
    flashback-point.  With FLAG_RELAXED off the basic condition applies."""
    if not (flags & FLAG_RELAXED):
        return basic_plan(prog, lv, p, c)
    if flags & FLAG_EXACT:
        from .exact import exact_plan_window
        return exact_plan_window(prog, lv, p, c, backups, flags)
    w = _Window(prog, lv, p, c, set(backups) if (flags & FLAG_OSRB) else set(), flags)
    w.sweep()
    if not (flags & FLAG_PRUNE) and not w.feasible():
        return None
    return w.plan()


def basic_plan(prog, lv, p, c):
    """Basic flashback condition: R_prec must not be overwritten by
    [I_prec, I_cur), and resume re-executes the window.  Feasible iff no
    register of LIVE_IN(p) is defined in W and every result-producing
    instruction in W can be re-executed (R-4).  S = LIVE_IN(p)."""
    W = range(p, c)
    ins = prog.instrs
    lin_p = lv.live_in[p]
    for j in W:
        r = ins[j].defreg
        if r is None:
            continue
        if r in lin_p or not reexec_op_kind(prog, ins[j]):
            return None
    w = _Window(prog, lv, p, c, set(), 0)
    for j in W:
        if ins[j].defreg is not None:
            w.reexec[j] = [w.supply_of(x) for x in w.opvals(j)]
            w.events.append(("X", j))
    S = {(r, PRE): "C" for r in lin_p}
    saved = sorted(((src, v) for v, src in S.items()), key=_saved_key)
    final = {}
    for r in sorted(lv.live_in[c]):
        d = w.rd(r, c)
        final[r] = ("X", d) if d is not PRE else ("C",)
    nb = _bytes_of(prog, S)
    nv = sum(1 for v in S if prog.is_vector(v[0]))
    return Plan(c, p, "basic", saved, [], list(w.events), dict(w.reexec), {}, final,
                nb, nv, len(S) - nv, 0, 0, len(w.reexec))


def live_plan(prog, lv, c):
    """LIVE (ref [4]): save LIVE_IN(c); flashback-point p = c."""
    w = _Window(prog, lv, c, c, set(), 0)
    pl = w.plan("live")
    return pl


def full_plan(prog, lv, c):
    """FULL_IR: every declared IR register, regardless of liveness (the
    analogue of the BASELINE routine that swaps all occupied resources)."""
    S = {(r, PRE): "C" for r in prog.all_regs()}
    saved = sorted(((src, v) for v, src in S.items()), key=_saved_key)
    final = {r: ("C",) for r in prog.all_regs()}
    nb = VEC_BYTES * prog.nv + SCA_BYTES * prog.ns
    return Plan(c, c, "full", saved, [], [], {}, {}, final, nb, prog.nv, prog.ns, 0, 0, 0)


@dataclass
class Analysis:
    prog: Program
    lv: Liveness
    sites: list
    heads: list
    backups: list                  # OSRB-selected scalar defs (global indices)
    plans: dict                    # site c -> chosen Plan
    live: dict                     # site c -> LIVE plan (fallback after a resume, R-16)
    candidates: dict = field(default_factory=dict)   # c -> {p: Plan or None}
    mode: int = MODE_CTXBACK
    flags: int = FLAGS_ALL
    defer: dict = field(default_factory=dict)        # site c -> site it defers to (c itself: none)


def resume_estimate(prog, pl, instr_bytes=DEFER_INSTR_BYTES, level_bytes=RESUME_LEVEL_BYTES):
    """FLAG_RANK_RESUME (NEXT N4; the paper ranks by preemption latency only
    and notes that re-execution can dominate resuming):
    estimated preempt + resume cost of a plan in context-byte units,

      E = 2 * payload                      context written at preempt, read at resume
        + sum of re-executed load bytes     128 B (vector) / 4 B (scalar) per warp
        + level_bytes * (levels - 1)        dependent memory round trips after the restore
        + instr_bytes * (#reverts + #re-executions)

    levels = depth of the resume schedule in memory round trips: a restored
    value (saved, backed up or recovered at preempt) is at level 1, a
    re-executed load at 1 + the deepest of its operands, any other re-executed
    or reverted instruction at the deepest of its operands."""
    saved_p = {(v[0], pl.revert_info[v][0]) for src, v in pl.saved if src == "P"}
    lx, lr = {}, {}

    def level(reg, s):
        if s[0] in ("C", "B"):
            return 1
        if s[0] == "X":
            return lx[s[1]]
        return 1 if (reg, s[1]) in saved_p else lr[(reg, s[1])]

    depth = 1 if pl.saved else 0
    load_bytes = 0
    for e in pl.schedule:
        if e[0] == "X":
            j = e[1]
            ins = prog.instrs[j]
            lv_ = max([level(r, s) for r, s in zip(ins.uses(), pl.reexec_supply[j])], default=0)
            if ins.op == "ldg":
                lv_ += 1
                load_bytes += VEC_BYTES if prog.is_vector(ins.defreg) else SCA_BYTES
            lx[j] = lv_
        else:
            v = e[1]
            m, _k, ins_, sups = pl.revert_info[v]
            lv_ = max([level(x[0], s) for x, s in zip(ins_, sups)], default=0)
            lr[(v[0], m)] = lv_
        depth = max(depth, lv_)
    ops = len(pl.schedule) + len(pl.preempt_reverts)
    return 2 * pl.payload_bytes + load_bytes + level_bytes * max(0, depth - 1) + instr_bytes * ops


def best_plan(prog, lv, heads, c, backups, flags, keep=None, est=None):
    """Enumerate p = c, c-1, ..., h(c) (R-1, R-3) and pick the lexicographic
    minimum of Plan.cost() (R-10); with FLAG_RANK_RESUME the minimum of
    (resume_estimate, Plan.cost()).  `est` = (instr_bytes, level_bytes)."""
    def key(pl):
        if flags & FLAG_RANK_RESUME:
            return (resume_estimate(prog, pl, *(est or ())),) + pl.cost()
        return pl.cost()
    best, best_k = None, None
    for p in range(c, heads[c] - 1, -1):
        pl = plan_window(prog, lv, p, c, backups, flags)
        if keep is not None:
            keep[p] = pl
        if pl is not None:
            k = key(pl)
            if best is None or k < best_k:
                best, best_k = pl, k
    return best


def osrb_candidates(prog):
    """R-7: irreversible scalar defs m whose old value is read in the same BB
    (by an instruction j <= m with no def of the register in [j, m))."""
    out = []
    for (s, e) in prog.bbs:
        for m in range(s, e):
            ins = prog.instrs[m]
            r = ins.defreg
            if r is None or r[0] != "s":
                continue
            if revert_spec(ins, r) is not None:
                continue
            read = r in ins.uses()
            j = m - 1
            while not read and j >= s:
                if prog.instrs[j].defreg == r:
                    break
                if r in prog.instrs[j].uses():
                    read = True
                j -= 1
            if read:
                out.append(m)
    return out


def defer_targets(prog, sites, plans, instr_bytes=DEFER_INSTR_BYTES):
    """CS-Defer and its combination with the site's own plan
    (P:325-329): a preemption arriving at site c may continue to a later site
    d of the same basic block (control flow must stay determinable) and
    save d's context there.  The paper ranks the options by estimated
    preemption latency and ignores the stalls of the in-between instructions
    (P:380); here E(c -> d) = bytes(plan at d) + instr_bytes * (d - c), and d
    minimises E over d >= c (ties: the earliest d, i.e. no deferral first)."""
    out = {}
    for c in sites:
        bb = prog.bb_of(c)
        best, best_e = c, None
        for d in sites:
            if d < c or prog.bb_of(d) != bb:
                continue
            e = plans[d].payload_bytes + instr_bytes * (d - c)
            if best_e is None or e < best_e:
                best, best_e = d, e
        out[c] = best
    return out


def analyze(prog: Program, policy="EVERY_INSTR", mode=MODE_CTXBACK, flags=FLAGS_ALL,
            every=8, sites=None, keep_candidates=False, defer_instr_bytes=DEFER_INSTR_BYTES,
            resume_level_bytes=RESUME_LEVEL_BYTES) -> Analysis:
    """Compile-time analysis: per poll site, the chosen plan."""
    an = _analyze(prog, policy, mode, flags & (FLAGS_ALL | FLAG_PRUNE | FLAG_RANK_RESUME | FLAG_EXACT), every, sites,
                  keep_candidates, (defer_instr_bytes, resume_level_bytes))
    an.flags = flags
    if flags & FLAG_DEFER:
        an.defer = defer_targets(prog, an.sites, an.plans, defer_instr_bytes)
    else:
        an.defer = {c: c for c in an.sites}
    return an


def _analyze(prog, policy, mode, flags, every, sites, keep_candidates, est=None):
    lv = liveness(prog)
    heads = region_heads(prog)
    if sites is None:
        sites = sites_for_policy(prog, policy, every)
    live = {c: live_plan(prog, lv, c) for c in sites}
    if mode == MODE_LIVE:
        return Analysis(prog, lv, sites, heads, [], dict(live), live, mode=mode, flags=flags)
    if mode == MODE_FULL:
        return Analysis(prog, lv, sites, heads, [], {c: full_plan(prog, lv, c) for c in sites},
                        live, mode=mode, flags=flags)
    backups = []
    if (flags & FLAG_OSRB) and (flags & FLAG_RELAXED):
        # R-7 selects backups by the bytes of the greedy R-10 choice, whatever
        # the ranking or the plan search (R-19)
        fb = flags & ~(FLAG_RANK_RESUME | FLAG_EXACT)
        base = {c: best_plan(prog, lv, heads, c, (), fb).payload_bytes for c in sites}
        for m in osrb_candidates(prog):
            bb = prog.bb_of(m)
            for c in sites:
                if prog.bb_of(c) != bb or c <= m or heads[c] > m:
                    continue
                if best_plan(prog, lv, heads, c, (m,), fb).payload_bytes < base[c]:
                    backups.append(m)
                    break
    plans, cands = {}, {}
    for c in sites:
        keep = {} if keep_candidates else None
        plans[c] = best_plan(prog, lv, heads, c, backups, flags, keep, est)
        if keep_candidates:
            cands[c] = keep
    return Analysis(prog, lv, sites, heads, backups, plans, live, cands, mode, flags)


def full_ir_bytes(prog):
    return VEC_BYTES * prog.nv + SCA_BYTES * prog.ns


def smem_slice(prog, warp):
    """Shared-memory words warp `warp` of a block saves / restores at a
    (block-uniform) barrier site: slice = ceil(smem / nwarps) words each."""
    if prog.smem == 0:
        return 0, 0
    sl = -(-prog.smem // prog.nwarps)
    lo = min(prog.smem, warp * sl)
    hi = min(prog.smem, lo + sl)
    return lo, hi


def plan_text(prog, pl: Plan) -> str:
    """Canonical one-line dump of a plan, for parity with the C++ analyzer."""
    def vs(v):
        r, d = v
        return f"{r}@{'PRE' if d is PRE else d}"

    def ss(s):
        return {"C": "C", "B": f"B{s[1] if len(s) > 1 else ''}", "X": f"X{s[1] if len(s) > 1 else ''}",
                "R": f"R{s[1] if len(s) > 1 else ''}"}[s[0]]
    parts = [f"c={pl.c}", f"p={pl.p}", f"bytes={pl.payload_bytes}", f"nv={pl.n_vec}", f"ns={pl.n_sca}"]
    parts.append("save=" + ",".join(f"{src}:{vs(v)}" for src, v in pl.saved))
    parts.append("pre=" + ",".join(f"{vs(e[0])}/m{e[1]}" for e in pl.preempt_reverts))
    sched = []
    for e in pl.schedule:
        if e[0] == "X":
            sched.append(f"X{e[1]}(" + ",".join(ss(s) for s in pl.reexec_supply[e[1]]) + ")")
        else:
            m, _k, _i, sups = pl.revert_info[e[1]]
            sched.append(f"R{vs(e[1])}/m{m}(" + ",".join(ss(s) for s in sups) + ")")
    parts.append("sched=" + ",".join(sched))
    parts.append("final=" + ",".join(f"{r}:{ss(s)}" for r, s in sorted(pl.final.items(),
                                                                     key=lambda t: (t[0][0] != 'v', int(t[0][1:])))))
    return " ".join(parts)
