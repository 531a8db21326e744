"""Exact minimum-bytes flashback plans (NEXT N4: "exact
min-bytes plan (ILP/BF) vs greedy"; reading R-19).

Test infrastructure only (see oracle/__init__.py).  Plain exhaustive search:
for a window W = [p, c) it enumerates the sets T of values that can be saved
at preemption and keeps the cheapest one whose resume closure yields every
required value.  The rules are the paper's, stated as a closure without the
CTXB-R1 sweep's order (the same statement as oracle/brute.py's BF2):

  obtainable at preempt:
      CURRENT values (still in their register at I_cur), OSRB backups of the
      selected scalar defs, and values recovered by reverting m = nd(r, d+1)
      from obtainable inputs (repeated until no change)
  resume closure of T:
      (def j, j) by re-executing a re-executable j (R-2, R-4) whose operand
      values are known; (r, d) by reverting m = nd(r, d+1) whose inputs
      (r, m) and m's other register operand values are known
  required (R-2): every live-out result of W and every pass-through
      value (r, PRE), r in LIVE_IN(c); with FLAG_PRUNE only the final value
      (r, rd(r, c)) of each r in LIVE_IN(c)

T minimises (bytes(T), |T|, T's candidate indices in canonical value order,
lexicographically).  The plan built from T: T's values are saved (CURRENT ->
'C', backup -> 'B', otherwise 'P' with its at-preempt revert chain); the
resume schedule is the establishment order of the closure (program-order
re-execution pass, then reverts in canonical value order, repeated), each
value keeping its first derivation, pruned to what the required values
demand.  p is then chosen by R-10 as for the greedy plans.

Search space reductions that cannot change the minimum or its tie-break:
candidates that are not *relevant* (neither required nor an input of a rule
whose output is relevant) are dropped; a *forced* candidate (without it even
all the others fall short) is in every feasible T; a candidate derivable from
the forced ones is in no minimal T.  Dropping keeps the canonical order of
the rest, and the forced values, common to every solution, do not affect
which of two solutions is lexicographically first.
"""
from __future__ import annotations

from itertools import combinations

from .analysis import (PRE, FLAG_OSRB, FLAG_PRUNE, FLAG_REVERT, Plan, VEC_BYTES, SCA_BYTES,
                       _Window, _saved_key, reexec_op_kind, revert_spec)

MAX_CANDIDATES = 18


class TooLarge(ValueError):
    """The window has more relevant candidate values than MAX_CANDIDATES."""


def vkey(prog, v):
    """Canonical value order: vectors before scalars, register index, PRE first."""
    r, d = v
    return (0 if prog.is_vector(r) else 1, int(r[1:]), -1 if d is PRE else d)


class ExactWindow:
    def __init__(self, prog, lv, p, c, backups, flags):
        self.prog, self.lv, self.p, self.c, self.flags = prog, lv, p, c, flags
        self.w = _Window(prog, lv, p, c, set(), 0)      # rd / nd / is_current / opvals only
        self.backups = sorted(m for m in backups if p <= m < c) if flags & FLAG_OSRB else []
        self.universe = sorted(self._all_values(), key=lambda v: vkey(prog, v))

    # -- the closure rules --------------------------------------------------------

    def _all_values(self):
        w, ins = self.w, self.prog.instrs
        regs, vals = set(self.lv.live_in[self.c]), set()
        for j in w.W:
            regs |= set(ins[j].uses())
            if ins[j].defreg:
                regs.add(ins[j].defreg)
                vals.add((ins[j].defreg, j))
        return vals | {(r, PRE) for r in regs}

    def revert_rule(self, v):
        """Alg. 2: (m, kind, inputs) recovering v = (r, d) by reverting
        m = nd(r, d+1), or None (R-5)."""
        if not (self.flags & FLAG_REVERT):
            return None
        r, d = v
        m = self.w.nd(r, self.p if d is PRE else d + 1)
        if m is None:
            return None
        spec = revert_spec(self.prog.instrs[m], r)
        if spec is None:
            return None
        kind, others = spec
        return m, kind, [(r, m)] + [(o.reg, self.w.rd(o.reg, m)) for o in others if o.is_reg]

    def reexec_ok(self, j):
        return self.w.reexec_kind(j)

    def required(self):
        w, ins = self.w, self.prog.instrs
        if self.flags & FLAG_PRUNE:
            return {(r, w.rd(r, self.c)) for r in self.lv.live_in[self.c]}
        req = {(ins[j].defreg, j) for j in w.W if w.liveout_def(j)}
        req |= {(r, PRE) for r in self.lv.live_in[self.c] if w.rd(r, self.c) is PRE}
        return req

    def preempt_derivations(self):
        """value -> ('C',) | ('B', m) | ('R', m, kind, inputs, supplies), first kept."""
        der = {}
        for v in self.universe:
            if self.w.is_current(v):
                der[v] = ("C",)
        for m in self.backups:
            s = self.prog.instrs[m].defreg
            v = (s, self.w.rd(s, m))
            if v not in der:
                der[v] = ("B", m)
        changed = True
        while changed:
            changed = False
            for v in self.universe:
                if v in der:
                    continue
                rule = self.revert_rule(v)
                if rule is None:
                    continue
                m, kind, inputs = rule
                if all(x in der for x in inputs):
                    der[v] = ("R", m, kind, inputs, [self._sup(der[x]) for x in inputs])
                    changed = True
        return der

    @staticmethod
    def _sup(d):
        return d if d[0] == "C" else (d[0], d[1])

    def closure(self, T):
        """Resume closure of the saved set T: (known, events, rev, reexec)."""
        ins = self.prog.instrs
        known = dict(T)                   # value -> supply
        events, rev, reexec = [], {}, {}
        changed = True
        while changed:
            changed = False
            for j in self.w.W:
                v = (ins[j].defreg, j)
                if j in reexec or v in known or not self.reexec_ok(j):
                    continue
                ov = self.w.opvals(j)
                if all(x in known for x in ov):
                    reexec[j] = [known[x] for x in ov]
                    known[v] = ("X", j)
                    events.append(("X", j))
                    changed = True
            for v in self.universe:
                if v in known:
                    continue
                rule = self.revert_rule(v)
                if rule is None:
                    continue
                m, kind, inputs = rule
                if all(x in known for x in inputs):
                    rev[v] = (m, kind, inputs, [known[x] for x in inputs])
                    known[v] = ("R", m)
                    events.append(("R", v))
                    changed = True
        return known, events, rev, reexec

    def relevant(self, req):
        """Values that are required or inputs of a rule producing a relevant value."""
        ins = self.prog.instrs
        rel = set(req)
        changed = True
        while changed:
            changed = False
            for j in self.w.W:
                if (ins[j].defreg, j) in rel and self.reexec_ok(j):
                    for x in self.w.opvals(j):
                        if x not in rel:
                            rel.add(x)
                            changed = True
            for v in list(rel):
                rule = self.revert_rule(v)
                if rule is not None:
                    for x in rule[2]:
                        if x not in rel:
                            rel.add(x)
                            changed = True
        return rel

    # -- the search -------------------------------------------------------------

    def minimum(self):
        """(T as a list of values in canonical order) or None if infeasible."""
        der = self.preempt_derivations()
        req = self.required()
        rel = self.relevant(req)
        cand = [v for v in self.universe if v in der and v in rel]
        full = {v: self._sup(der[v]) for v in cand}
        if not req <= set(self.closure(full)[0]):
            return None
        # forced: without it even all the other candidates fall short, so it is
        # in every feasible T (and, common to all, does not affect the order of
        # the rest); a candidate derivable from the forced ones is in no minimal T
        forced = [v for v in cand
                  if not req <= set(self.closure({u: full[u] for u in cand if u != v})[0])]
        known_f = self.closure({u: full[u] for u in forced})[0]
        rest = [v for v in cand if v not in forced and v not in known_f]
        if len(rest) > MAX_CANDIDATES:
            raise TooLarge(f"{len(rest)} candidate values")
        size = [VEC_BYTES if self.prog.is_vector(v[0]) else SCA_BYTES for v in rest]
        base = sum(VEC_BYTES if self.prog.is_vector(v[0]) else SCA_BYTES for v in forced)
        best = None                        # ((bytes, k), T)
        for k in range(len(rest) + 1):
            for T in combinations(range(len(rest)), k):
                key = (base + sum(size[i] for i in T), len(forced) + k)
                if best is not None and key >= best[0]:
                    continue
                sel = {u: full[u] for u in forced}
                sel.update({rest[i]: full[rest[i]] for i in T})
                if req <= set(self.closure(sel)[0]):
                    best = (key, T)
        return sorted(forced + [rest[i] for i in best[1]], key=lambda v: vkey(self.prog, v))

    def plan(self):
        T = self.minimum()
        if T is None:
            return None
        der = self.preempt_derivations()
        prog, ins = self.prog, self.prog.instrs
        saved_src, Tsup = {}, {}
        for v in T:
            d = der[v]
            saved_src[v] = {"C": "C", "B": "B", "R": "P"}[d[0]]
            Tsup[v] = self._sup(d)
        known, events, rev, reexec = self.closure(Tsup)
        # demand-driven pruning from the required values
        used_x, used_res, used_pre, S = set(), set(), set(), {}

        def pre(v):
            if v in used_pre:
                return
            used_pre.add(v)
            for x, s in zip(der[v][3], der[v][4]):
                if s[0] == "R":
                    pre(x)

        def demand(v):
            if v in Tsup:
                S[v] = saved_src[v]
                if saved_src[v] == "P":
                    pre(v)
                return
            s = known[v]
            if s[0] == "X":
                if s[1] not in used_x:
                    used_x.add(s[1])
                    for x in self.w.opvals(s[1]):
                        demand(x)
            elif v not in used_res:
                used_res.add(v)
                for x in rev[v][2]:
                    demand(x)
        for v in sorted(self.required(), key=lambda x: vkey(prog, x)):
            demand(v)
        assert set(S) == set(T), "a minimal saved set is fully demanded"
        saved = sorted(((src, v) for v, src in S.items()), key=_saved_key)
        pre_list = sorted(used_pre, key=lambda x: -der[x][1])
        preempt_reverts = [(v,) + tuple(der[v][1:]) for v in pre_list]
        schedule = [e for e in events
                    if (e[0] == "X" and e[1] in used_x) or (e[0] == "R" and e[1] in used_res)]
        # an intermediate of an at-preempt chain may also be re-derived at
        # resume (with resume-time supplies): the resume record wins here,
        # the preempt record travels in preempt_reverts
        revert_info = {v: tuple(der[v][1:]) for v in used_pre}
        revert_info.update({v: rev[v] for v in used_res})
        final = {}
        for r in sorted(self.lv.live_in[self.c]):
            d = self.w.rd(r, self.c)
            final[r] = known[(r, d)] if d is not PRE else ("C",)
        nb = sum(VEC_BYTES if prog.is_vector(v[0]) else SCA_BYTES for v in S)
        nv = sum(1 for v in S if prog.is_vector(v[0]))
        bkp = {v: der[v][1] for v in S if S[v] == "B"}
        return Plan(self.c, self.p, "ctxback", saved, preempt_reverts, schedule,
                    {j: reexec[j] for j in used_x}, revert_info, final, nb, nv, len(S) - nv,
                    len(used_pre), len(used_res), len(used_x), bkp)


def exact_plan_window(prog, lv, p, c, backups=(), flags=0):
    return ExactWindow(prog, lv, p, c, backups, flags).plan()
