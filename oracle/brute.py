"""Brute-force checks of the flashback analysis on tiny kernels (BF1-BF3).

Test infrastructure only.  Independent of the CTXB-R1 sweep's order-dependent
details: it states the relaxed condition and the availability rules
of Alg. 2 as a plain closure and enumerates saved sets.

BF2 (exhaustive minimum): the values obtainable on chip at preempt time are
  * CURRENT values (still in their register at I_cur),
  * OSRB backups of selected scalar defs,
  * values recoverable by reverting with inputs obtainable at preempt.
For every subset T of them, the resume closure adds
  * (def j, j) for a re-executable j whose operand values are all known,
  * (r, d) by reverting m = next def of r when (r, m) and m's other operand
    values are known.
T is feasible iff the closure contains every live-out result of the window
(R-2) and every pass-through live-in value of I_cur.  BF-min is the
least bytes over feasible T.  Any correct plan's saved set is such a T, so
plan bytes >= BF-min, and oracle-feasible => BF-feasible.
"""
from __future__ import annotations

from itertools import combinations

from .analysis import (PRE, VEC_BYTES, SCA_BYTES, _Window, reexec_op_kind, revert_spec,
                       plan_window)


def _vbytes(v):
    return VEC_BYTES if v[0][0] == "v" else SCA_BYTES


class BFWindow:
    def __init__(self, prog, lv, p, c, backups=()):
        self.w = _Window(prog, lv, p, c, set(), 0)
        self.prog, self.lv, self.p, self.c = prog, lv, p, c
        self.backups = [m for m in backups if p <= m < c]

    def _revert_inputs(self, v):
        w = self.w
        r, d = v
        m = w.nd(r, self.p if d is PRE else d + 1)
        if m is None:
            return None
        spec = revert_spec(self.prog.instrs[m], r)
        if spec is None:
            return None
        return [(r, m)] + [(o.reg, w.rd(o.reg, m)) for o in spec[1] if o.is_reg]

    def all_values(self):
        """Every value (r, d) of the window that any computation can refer to."""
        w = self.w
        vals = set()
        regs = set()
        for j in w.W:
            ins = self.prog.instrs[j]
            regs |= set(ins.uses())
            if ins.defreg:
                regs.add(ins.defreg)
                vals.add((ins.defreg, j))
        regs |= set(self.lv.live_in[self.c])
        for r in regs:
            vals.add((r, PRE))
        return vals

    def preempt_obtainable(self):
        w = self.w
        base = {v for v in self.all_values() if w.is_current(v)}
        for m in self.backups:
            s = self.prog.instrs[m].defreg
            base.add((s, w.rd(s, m)))
        known = set(base)
        changed = True
        while changed:
            changed = False
            for v in self.all_values():
                if v in known:
                    continue
                ins_ = self._revert_inputs(v)
                if ins_ is not None and all(x in known for x in ins_):
                    known.add(v)
                    changed = True
        return known

    def required(self):
        w = self.w
        req = set()
        for j in w.W:
            if w.liveout_def(j):
                req.add((self.prog.instrs[j].defreg, j))
        for r in self.lv.live_in[self.c]:
            if w.rd(r, self.c) is PRE:
                req.add((r, PRE))
        return req

    def closure(self, T):
        w = self.w
        known = set(T)
        allv = self.all_values()
        changed = True
        while changed:
            changed = False
            for j in w.W:
                ins = self.prog.instrs[j]
                v = (ins.defreg, j)
                if ins.defreg is None or v in known:
                    continue
                if w.liveout_def(j) and reexec_op_kind(self.prog, ins) and \
                        all(x in known for x in w.opvals(j)):
                    known.add(v)
                    changed = True
            for v in allv:
                if v in known:
                    continue
                ins_ = self._revert_inputs(v)
                if ins_ is not None and all(x in known for x in ins_):
                    known.add(v)
                    changed = True
        return known

    def feasible_set(self, T):
        return self.required() <= self.closure(T)

    def minimum(self, max_values=16):
        """Exhaustive BF-min over subsets of the preempt-obtainable values
        (smallest byte count first).  Returns (bytes, T) or None."""
        cand = sorted(self.preempt_obtainable(), key=lambda v: (v[0], -1 if v[1] is PRE else v[1]))
        if len(cand) > max_values:
            raise ValueError("too many candidate values for brute force")
        best = None
        req = self.required()
        for k in range(len(cand) + 1):
            for T in combinations(cand, k):
                b = sum(_vbytes(v) for v in T)
                if best is not None and b >= best[0]:
                    continue
                if req <= self.closure(T):
                    best = (b, set(T))
        return best


def plan_saved_values(pl):
    return {v for _src, v in pl.saved}


def check_window(prog, lv, p, c, backups=(), flags=7):
    """BF2 for one (c, p): returns dict(oracle_bytes, bf_bytes, oracle_feasible,
    bf_feasible, sound)."""
    pl = plan_window(prog, lv, p, c, backups, flags)
    bf = BFWindow(prog, lv, p, c, backups if (flags & 4) else ())
    mn = bf.minimum()
    out = dict(oracle_feasible=pl is not None, bf_feasible=mn is not None,
               oracle_bytes=pl.payload_bytes if pl else None, bf_bytes=mn[0] if mn else None)
    if pl is not None:
        S = plan_saved_values(pl)
        out["sound"] = bf.feasible_set(S) and S <= bf.preempt_obtainable()
    return out
