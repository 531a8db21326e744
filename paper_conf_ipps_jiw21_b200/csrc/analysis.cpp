// Compile-time flashback analysis in the normative reading CTXB-R1
// (SURVEY §8(c2)).  Paper passages:
//   liveness = register context of an instruction .................. P:80
//   window [I_prec, I_cur), signal handled before I_cur ............. P:74 (R-1)
//   relaxed condition, Alg. 1 ....................................... P:88-152 (R-2)
//   instruction reverting, Alg. 2 ................................... P:154-231 (R-5, R-6)
//   on-chip scalar register backup .................................. P:257-269 (R-7)
//   combined fixpoint ............................................... P:271-303 (R-9)
//   windows inside the basic block and idempotent region ............ P:305 (R-3)
//   least-latency flashback-point per instruction ................... P:313, P:337 (R-10)
//   context incl. results restored by saving/reloading .............. P:343 (R-8)
#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <exception>
#include <functional>
#include <set>
#include <sstream>
#include <thread>

#include "ctxb_internal.h"

namespace ctxb {
namespace {

constexpr uint32_t F_RELAXED = 1, F_REVERT = 2, F_OSRB = 4, F_DEFER = 8, F_PRUNE = 16, F_RANK_RESUME = 32,
                   F_EXACT = 64;
constexpr uint32_t VEC_B = 128, SCA_B = 4;

bool is_alu(Op o) {
  switch (o) {
    case Op::Mov: case Op::Not: case Op::Neg: case Op::I2F: case Op::U2F: case Op::F2I:
    case Op::IAdd: case Op::ISub: case Op::IMul: case Op::And: case Op::Or: case Op::Xor:
    case Op::Shl: case Op::Shr: case Op::Sar: case Op::RotL: case Op::RotR: case Op::UMin:
    case Op::UMax: case Op::IMin: case Op::IMax: case Op::FAdd: case Op::FSub: case Op::FMul:
    case Op::FFma: case Op::IMad: case Op::Sel: case Op::Setp:
      return true;
    default:
      return false;
  }
}

// R-4: ALU ops and loads from read-only buffers can be re-executed (not loads
// from rw buffers or shared memory, which other warps write).
bool reexec_op(const Program& P, const Instr& I) {
  if (is_alu(I.op)) return true;
  if (I.op == Op::Ldg) return P.buf_kinds[I.buf] == B_RO;
  return false;
}

int regid(const Program& P, const Operand& o) { return o.kind == OK::V ? (int)o.val : P.nv + (int)o.val; }

// R-5: r' = op(r, {R}) with a bit-exact inverse.  Fills kind and the
// non-shared operands (in operand order).
bool revert_spec(const Program& P, const Instr& I, int r, RevKind* kind, std::vector<Operand>* others) {
  if (I.defreg != r || I.dst.kind == OK::None) return false;
  if (I.guard.kind != OK::None || I.idx.kind != OK::None) return false;
  int cnt = 0;
  for (auto& o : I.srcs)
    if (o.is_reg() && regid(P, o) == r) cnt++;
  if (cnt != 1) return false;
  others->clear();
  if (I.op == Op::Not || I.op == Op::Neg) {
    *kind = I.op == Op::Not ? RV_NOT_D : RV_NEG_D;
    return true;
  }
  if (I.srcs.size() != 2) return false;
  const Operand& a = I.srcs[0];
  const Operand& b = I.srcs[1];
  bool a_is = a.is_reg() && regid(P, a) == r;
  const Operand& other = a_is ? b : a;
  switch (I.op) {
    case Op::IAdd: *kind = RV_SUB_D; others->push_back(other); return true;
    case Op::ISub:
      *kind = a_is ? RV_ADD_D : RV_RSUB_D;
      others->push_back(other);
      return true;
    case Op::Xor: *kind = RV_XOR_D; others->push_back(other); return true;
    case Op::IMul:
      if (other.kind == OK::Imm && (other.val & 1u)) {
        *kind = RV_MULINV;
        others->push_back(other);
        return true;
      }
      return false;
    case Op::RotL: case Op::RotR:
      if (a_is && b.kind == OK::Imm) {
        *kind = I.op == Op::RotL ? RV_ROTR : RV_ROTL;
        others->push_back(b);
        return true;
      }
      return false;
    default:
      return false;
  }
}

struct Liveness {
  std::vector<std::vector<uint8_t>> in, out;
};

Liveness liveness(const Program& P) {
  int R = P.nregs(), nb = (int)P.bbs.size();
  std::vector<std::vector<uint8_t>> use(nb, std::vector<uint8_t>(R, 0)), def(nb, std::vector<uint8_t>(R, 0)),
      lin(nb, std::vector<uint8_t>(R, 0)), lout(nb, std::vector<uint8_t>(R, 0));
  for (int b = 0; b < nb; b++)
    for (int i = P.bbs[b].first; i < P.bbs[b].second; i++) {
      for (int u : P.ins[i].uses)
        if (!def[b][u]) use[b][u] = 1;
      if (P.ins[i].defreg >= 0) def[b][P.ins[i].defreg] = 1;
    }
  bool changed = true;
  while (changed) {
    changed = false;
    for (int b = nb - 1; b >= 0; b--) {
      std::vector<uint8_t> o(R, 0), i_(R, 0);
      for (int s : P.succ[b])
        for (int r = 0; r < R; r++) o[r] |= lin[s][r];
      for (int r = 0; r < R; r++) i_[r] = use[b][r] | (o[r] & !def[b][r]);
      if (o != lout[b] || i_ != lin[b]) {
        lout[b] = o;
        lin[b] = i_;
        changed = true;
      }
    }
  }
  Liveness L;
  int n = (int)P.ins.size();
  L.in.assign(n, {});
  L.out.assign(n, {});
  for (int b = 0; b < nb; b++) {
    std::vector<uint8_t> cur = lout[b];
    for (int i = P.bbs[b].second - 1; i >= P.bbs[b].first; i--) {
      L.out[i] = cur;
      if (P.ins[i].defreg >= 0) cur[P.ins[i].defreg] = 0;
      for (int u : P.ins[i].uses) cur[u] = 1;
      L.in[i] = cur;
    }
  }
  return L;
}

// h(c): max(BB start, idempotent-region start); a region starts after every
// atomic and at a store to a buffer loaded earlier in the region (R-3).
std::vector<int> region_heads(const Program& P) {
  std::vector<int> heads(P.ins.size(), 0);
  for (auto [s, e] : P.bbs) {
    int head = s;
    std::set<int> loaded;
    for (int c = s; c < e; c++) {
      heads[c] = head;
      const Instr& I = P.ins[c];
      const int SMEM_BUF = -2;   // shared memory as one more buffer for the WAR rule
      if (I.op == Op::AtomAdd || I.op == Op::AtomCas || I.op == Op::Bar) {
        head = c + 1;
        loaded.clear();
      } else if ((I.op == Op::Stg && loaded.count(I.buf)) || (I.op == Op::Sts && loaded.count(SMEM_BUF))) {
        head = c;
        loaded.clear();
      } else if (I.op == Op::Ldg) {
        loaded.insert(I.buf);
      } else if (I.op == Op::Lds) {
        loaded.insert(SMEM_BUF);
      }
    }
  }
  return heads;
}

std::vector<int> sites_for(const Program& P, const Options& opt) {
  std::vector<int> out;
  if (P.has_barriers && opt.policy != 2) {   // block-uniform preemption, fused with the barriers (N2)
    for (int i = 0; i < (int)P.ins.size(); i++)
      if (P.ins[i].op == Op::Bar) out.push_back(i);
    return out;
  }
  if (opt.policy == 0) {
    for (int i = 0; i < (int)P.ins.size(); i++) out.push_back(i);
  } else if (opt.policy == 2) {
    std::set<int> s(P.explicit_sites.begin(), P.explicit_sites.end());
    out.assign(s.begin(), s.end());
  } else {
    int N = (int)std::max<uint32_t>(1, opt.every);
    std::set<int> s;
    for (int b = 0; b < (int)P.bbs.size(); b++) {
      auto [s0, e0] = P.bbs[b];
      for (int i = s0 + N; i < e0; i += N) s.insert(i);
      const Instr& last = P.ins[e0 - 1];
      if ((last.op == Op::Bra || last.op == Op::Brnz || last.op == Op::Brz) && last.target_bb <= b) s.insert(e0 - 1);
    }
    out.assign(s.begin(), s.end());
  }
  return out;
}

struct Deriv {
  SK k = SK::C;
  int arg = -1;
  bool present = false;
};

// Per-BB sorted definition positions of every register.
struct DefIndex {
  std::vector<std::vector<std::vector<int>>> pos;  // [bb][reg] -> positions
  explicit DefIndex(const Program& P) {
    pos.assign(P.bbs.size(), std::vector<std::vector<int>>(P.nregs()));
    for (int i = 0; i < (int)P.ins.size(); i++)
      if (P.ins[i].defreg >= 0) pos[P.bb_of[i]][P.ins[i].defreg].push_back(i);
  }
};

// One (site c, flashback-point p) evaluation of the CTXB-R1 sweep.
class Window {
 public:
  Window(const Program& P, const Liveness& L, const DefIndex& D, int p, int c, const std::vector<int>& backups,
         uint32_t flags)
      : P(P), L(L), D(D), p(p), c(c), flags(flags) {
    bb = P.bb_of[std::min(c, (int)P.ins.size() - 1)];
    if (c > p) bb = P.bb_of[p];
    int R = P.nregs();
    vpre.assign(R, {});
    vdef.assign(c - p, {});
    reexec.assign(c - p, 0);
    for (int r = 0; r < R; r++) set_valid({r, rd(r, c)}, {SK::C, -1, true});
    std::vector<int> bs(backups);
    std::sort(bs.begin(), bs.end());
    for (int m : bs)
      if (p <= m && m < c) {
        int s = P.ins[m].defreg;
        Val v{s, rd(s, m)};
        if (!valid(v)) set_valid(v, {SK::B, m, true});
      }
  }

  int rd(int r, int t) const {  // last def of r in [p, t), else PRE
    if (t <= p) return PRE;
    const auto& v = D.pos[P.bb_of[p < (int)P.ins.size() ? p : t - 1]][r];
    auto it = std::lower_bound(v.begin(), v.end(), t);
    if (it == v.begin()) return PRE;
    --it;
    return *it >= p ? *it : PRE;
  }
  int nd(int r, int t) const {  // first def of r in [t, c), else -1
    if (t >= c) return -1;
    const auto& v = D.pos[P.bb_of[t]][r];
    auto it = std::lower_bound(v.begin(), v.end(), t);
    if (it == v.end() || *it >= c) return -1;
    return *it;
  }
  bool is_current(const Val& v) const { return nd(v.r, v.d == PRE ? p : v.d + 1) < 0; }
  bool valid(const Val& v) const { return v.d == PRE ? vpre[v.r].present : vdef[v.d - p].present; }
  const Deriv& deriv(const Val& v) const { return v.d == PRE ? vpre[v.r] : vdef[v.d - p]; }
  void set_valid(const Val& v, Deriv d) {
    d.present = true;
    if (v.d == PRE)
      vpre[v.r] = d;
    else
      vdef[v.d - p] = d;
  }
  std::vector<Val> opvals(int j) const {
    std::vector<Val> out;
    for (int u : P.ins[j].uses) out.push_back({u, rd(u, j)});
    return out;
  }
  bool liveout_def(int j) const {
    int r = P.ins[j].defreg;
    return r >= 0 && L.out[j][r];
  }
  bool reexec_kind(int j) const { return liveout_def(j) && reexec_op(P, P.ins[j]); }
  Supply to_supply(const Deriv& d) const { return {d.k, d.arg}; }
  Supply supply_of(const Val& v) const {
    if (v.d != PRE && reexec[v.d - p]) return {SK::X, v.d};
    return to_supply(deriv(v));
  }

  bool try_revert(const Val& v) {
    if (!(flags & F_REVERT)) return false;
    int m = nd(v.r, v.d == PRE ? p : v.d + 1);
    if (m < 0) return false;
    RevertRec rec;
    if (!revert_spec(P, P.ins[m], v.r, &rec.kind, &rec.others)) return false;
    rec.v = v;
    rec.m = m;
    rec.inputs.push_back({v.r, m});
    for (auto& o : rec.others)
      if (o.is_reg()) {
        int u = regid(P, o);
        rec.inputs.push_back({u, rd(u, m)});
      }
    for (auto& x : rec.inputs) {
      if (is_current(x)) {
        rec.supplies.push_back({SK::C, -1});
      } else if (valid(x)) {
        rec.supplies.push_back(supply_of(x));
      } else if (try_revert(x)) {
        rec.supplies.push_back(to_supply(deriv(x)));
      } else {
        return false;
      }
    }
    set_valid(v, {SK::R, m, true});
    revs[v] = rec;
    events.push_back({false, m, v});
    return true;
  }

  void sweep() {
    bool changed = true;
    while (changed) {
      changed = false;
      for (int j = p; j < c; j++) {
        if (reexec[j - p] || !reexec_kind(j)) continue;
        auto ov = opvals(j);
        for (auto& x : ov)
          if (!valid(x) && try_revert(x)) changed = true;
        bool all = true;
        for (auto& x : ov) all = all && valid(x);
        if (all) {
          std::vector<Supply> sup;
          for (auto& x : ov) sup.push_back(supply_of(x));
          reexec[j - p] = 1;
          rx_supply[j] = sup;
          events.push_back({true, j, {P.ins[j].defreg, j}});
          Val v{P.ins[j].defreg, j};
          if (!valid(v)) set_valid(v, {SK::X, j, true});
          changed = true;
        }
      }
      for (int j = p; j < c; j++)
        if (liveout_def(j)) {
          Val v{P.ins[j].defreg, j};
          if (!valid(v) && try_revert(v)) changed = true;
        }
    }
  }

  bool feasible() const {
    for (int j = p; j < c; j++)
      if (liveout_def(j) && !valid({P.ins[j].defreg, j})) return false;
    return true;
  }

  // Resume-time demands.  R-2 (literal): every re-executed instruction's
  // operands and every live-out result of the window.  F_PRUNE (demand-driven
  // restore): only the final value of each register live-in at I_cur;
  // re-executions are then demanded transitively in compute_S.
  std::vector<std::pair<Val, Supply>> demands() const {
    std::vector<std::pair<Val, Supply>> out;
    if (flags & F_PRUNE) {
      for (int r = 0; r < P.nregs(); r++)
        if (L.in[c][r]) {
          int d = rd(r, c);
          out.push_back({{r, d}, d == PRE ? Supply{SK::C, -1} : supply_of({r, d})});
        }
      return out;
    }
    for (int j = p; j < c; j++)
      if (reexec[j - p]) {
        auto ov = opvals(j);
        const auto& sup = rx_supply.at(j);
        for (size_t k = 0; k < ov.size(); k++) out.push_back({ov[k], sup[k]});
      }
    for (int j = p; j < c; j++)
      if (liveout_def(j) && !reexec[j - p]) {
        Val v{P.ins[j].defreg, j};
        out.push_back({v, to_supply(deriv(v))});
      }
    for (int r = 0; r < P.nregs(); r++)
      if (L.in[c][r] && rd(r, c) == PRE) out.push_back({{r, PRE}, {SK::C, -1}});
    return out;
  }

  struct SRes {
    std::map<Val, char> S;
    std::set<Val> used_res, used_pre;
    std::set<int> used_x;   // re-executions the demands reach (all of them without F_PRUNE)
  };

  SRes compute_S(const std::map<Val, char>& pos) const {
    SRes R;
    std::function<void(const Val&)> pre_closure = [&](const Val& v) {
      if (R.used_pre.count(v)) return;
      R.used_pre.insert(v);
      const RevertRec& rec = revs.at(v);
      for (size_t k = 0; k < rec.inputs.size(); k++)
        if (rec.supplies[k].k == SK::R) pre_closure(rec.inputs[k]);
    };
    std::function<void(const Val&, const Supply&)> demand = [&](const Val& v, const Supply& s) {
      switch (s.k) {
        case SK::C: R.S.emplace(v, 'C'); break;
        case SK::B: R.S.emplace(v, 'B'); break;
        case SK::X:
          if ((flags & F_PRUNE) && !R.used_x.count(s.arg)) {
            R.used_x.insert(s.arg);
            auto ov = opvals(s.arg);
            const auto& sup = rx_supply.at(s.arg);
            for (size_t k = 0; k < ov.size(); k++) demand(ov[k], sup[k]);
          }
          break;
        case SK::R: {
          auto it = pos.find(v);
          char ps = it == pos.end() ? 'R' : it->second;
          if (ps == 'P') {
            R.S.emplace(v, 'P');
            pre_closure(v);
          } else {
            if (R.used_res.count(v)) return;
            R.used_res.insert(v);
            const RevertRec& rec = revs.at(v);
            for (size_t k = 0; k < rec.inputs.size(); k++) demand(rec.inputs[k], rec.supplies[k]);
          }
          break;
        }
      }
    };
    for (auto& [v, s] : demands()) demand(v, s);
    if (!(flags & F_PRUNE))
      for (int j = p; j < c; j++)
        if (reexec[j - p]) R.used_x.insert(j);
    return R;
  }

  uint32_t bytes_of(const std::map<Val, char>& S) const {
    uint32_t b = 0;
    for (auto& [v, src] : S) b += P.is_vec(v.r) ? VEC_B : SCA_B;
    return b;
  }

  Plan plan(int kind) const {
    std::map<Val, char> pos;
    for (auto& [v, rec] : revs) pos[v] = 'R';
    SRes r0 = compute_S(pos);
    std::vector<Val> order(r0.used_res.begin(), r0.used_res.end());
    std::stable_sort(order.begin(), order.end(),
                     [&](const Val& a, const Val& b) { return revs.at(a).m > revs.at(b).m; });
    for (const Val& v : order) {
      const RevertRec& rec = revs.at(v);
      bool forced = false;
      for (size_t k = 0; k < rec.inputs.size(); k++) {
        const Supply& s = rec.supplies[k];
        if (s.k == SK::X || (s.k == SK::R && pos.at(rec.inputs[k]) == 'R')) forced = true;
      }
      if (forced) continue;
      pos[v] = 'P';
      uint32_t bP = bytes_of(compute_S(pos).S);
      pos[v] = 'R';
      uint32_t bR = bytes_of(compute_S(pos).S);
      if (bP < bR) pos[v] = 'P';
    }
    SRes fin = compute_S(pos);
    Plan pl;
    pl.valid = true;
    pl.c = c;
    pl.p = p;
    pl.kind = kind;
    for (auto& [v, src] : fin.S) {
      SavedVal sv{src, v, -1};
      if (src == 'B') sv.bkp_m = deriv(v).arg;
      pl.saved.push_back(sv);
    }
    std::sort(pl.saved.begin(), pl.saved.end(), [](const SavedVal& a, const SavedVal& b) {
      if (a.v.r != b.v.r) return a.v.r < b.v.r;
      if (a.v.d != b.v.d) return a.v.d < b.v.d;
      return a.src < b.src;
    });
    std::vector<Val> pre(fin.used_pre.begin(), fin.used_pre.end());
    std::stable_sort(pre.begin(), pre.end(), [&](const Val& a, const Val& b) { return revs.at(a).m > revs.at(b).m; });
    for (auto& v : pre) pl.pre_reverts.push_back(revs.at(v));
    for (auto& e : events)
      if ((e.is_x && fin.used_x.count(e.j)) || (!e.is_x && fin.used_res.count(e.v))) pl.schedule.push_back(e);
    for (int j : fin.used_x) pl.reexec_supply[j] = rx_supply.at(j);
    pl.revert_info = revs;
    for (int r = 0; r < P.nregs(); r++)
      if (L.in[c][r]) {
        int d = rd(r, c);
        pl.final_.push_back({r, d == PRE ? Supply{SK::C, -1} : supply_of({r, d})});
      }
    pl.payload_bytes = bytes_of(fin.S);
    for (auto& [v, src] : fin.S) (P.is_vec(v.r) ? pl.n_vec : pl.n_sca)++;
    pl.n_rev_pre = (uint32_t)fin.used_pre.size();
    pl.n_rev_res = (uint32_t)fin.used_res.size();
    pl.n_reexec = (uint32_t)fin.used_x.size();
    return pl;
  }

  const Program& P;
  const Liveness& L;
  const DefIndex& D;
  int p, c, bb;
  uint32_t flags;
  std::vector<Deriv> vpre, vdef;
  std::vector<uint8_t> reexec;
  std::map<int, std::vector<Supply>> rx_supply;
  std::map<Val, RevertRec> revs;
  std::vector<Event> events;
};

// Basic condition: R_prec not overwritten in [I_prec, I_cur) and
// every result-producing instruction re-executable; S = LIVE_IN(p).
Plan basic_plan(const Program& P, const Liveness& L, const DefIndex& D, int p, int c) {
  for (int j = p; j < c; j++) {
    int r = P.ins[j].defreg;
    if (r < 0) continue;
    if (L.in[p][r] || !reexec_op(P, P.ins[j])) return Plan{};
  }
  Window w(P, L, D, p, c, {}, 0);
  for (int j = p; j < c; j++)
    if (P.ins[j].defreg >= 0) {
      std::vector<Supply> sup;
      for (auto& x : w.opvals(j)) sup.push_back(w.supply_of(x));
      w.reexec[j - p] = 1;
      w.rx_supply[j] = sup;
      w.events.push_back({true, j, {P.ins[j].defreg, j}});
    }
  Plan pl;
  pl.valid = true;
  pl.c = c;
  pl.p = p;
  pl.kind = 3;
  for (int r = 0; r < P.nregs(); r++)
    if (L.in[p][r]) {
      pl.saved.push_back({'C', {r, PRE}, -1});
      (P.is_vec(r) ? pl.n_vec : pl.n_sca)++;
      pl.payload_bytes += P.is_vec(r) ? VEC_B : SCA_B;
    }
  pl.schedule = w.events;
  pl.reexec_supply = w.rx_supply;
  for (int r = 0; r < P.nregs(); r++)
    if (L.in[c][r]) {
      int d = w.rd(r, c);
      pl.final_.push_back({r, d == PRE ? Supply{SK::C, -1} : Supply{SK::X, d}});
    }
  pl.n_reexec = (uint32_t)w.rx_supply.size();
  return pl;
}

// ---- CTXB_EXACT (NEXT N4 "exact min-bytes plan vs greedy"; R-19) ---
// The paper's rules as an order-free closure: T = values saved at preempt
// (CURRENT, OSRB backups, or recovered there by reverting, P:92, P:180,
// P:265); at resume, re-execute a re-executable j whose operand values are
// known (R-2, R-4) or revert m = nd(r, d+1) whose inputs are known
// (P:222-229).  Among the T whose closure holds every required value (R-2:
// live-out results of W + pass-through live-ins; F_PRUNE: final values of
// LIVE_IN(c)), pick the minimum of (bytes, |T|, T's candidate indices in value
// order).  Branch and bound, include-first in value order (so the first of
// several equal keys found is the lexicographically first), with the greedy
// plan's key as the initial bound and a node budget; a window whose search
// runs out of budget keeps its greedy plan (counted as truncated).
struct ExactCfg {
  uint32_t budget = 1u << 20;   // search nodes per window
  uint32_t max_cand = 48;       // relevant candidates beyond which the search is skipped
  uint32_t windows = 0, truncated = 0, improved = 0, fallback = 0;
};

class ExactWin {
 public:
  ExactWin(const Program& P, const Liveness& L, const DefIndex& D, int p, int c, const std::vector<int>& bk,
           uint32_t flags)
      : P(P), L(L), w(P, L, D, p, c, {}, 0), p(p), c(c), flags(flags) {
    std::set<int> regs;
    std::set<Val> vals;
    for (int r = 0; r < P.nregs(); r++)
      if (L.in[c][r]) regs.insert(r);
    for (int j = p; j < c; j++) {
      for (int u : P.ins[j].uses) regs.insert(u);
      if (P.ins[j].defreg >= 0) {
        regs.insert(P.ins[j].defreg);
        vals.insert({P.ins[j].defreg, j});
      }
    }
    for (int r : regs) vals.insert({r, PRE});
    U.assign(vals.begin(), vals.end());   // canonical order: register id, then PRE, then position
    for (size_t i = 0; i < U.size(); i++) idx[U[i]] = (int)i;
    if (flags & F_OSRB)
      for (int m : bk)
        if (p <= m && m < c) backups.push_back(m);
    std::sort(backups.begin(), backups.end());
    // rules: re-executions (program order), then reverts (value order)
    for (int j = p; j < c; j++)
      if (w.reexec_kind(j)) {
        Rule R;
        R.out = idx.at({P.ins[j].defreg, j});
        R.j = j;
        for (auto& x : w.opvals(j)) R.in.push_back(idx.at(x));
        xr.push_back(R);
      }
    for (size_t i = 0; i < U.size(); i++) {
      RevertRec rec;
      if (!revert_rule(U[i], &rec)) continue;
      Rule R;
      R.out = (int)i;
      R.j = rec.m;
      for (auto& x : rec.inputs) R.in.push_back(idx.at(x));
      rr.push_back(R);
      rrec[(int)i] = rec;
    }
    for (size_t k = 0; k < xr.size(); k++) xr_of_out[xr[k].out] = (int)k;
  }

  bool revert_rule(const Val& v, RevertRec* rec) const {
    if (!(flags & F_REVERT)) return false;
    int m = w.nd(v.r, v.d == PRE ? p : v.d + 1);
    if (m < 0) return false;
    if (!revert_spec(P, P.ins[m], v.r, &rec->kind, &rec->others)) return false;
    rec->v = v;
    rec->m = m;
    rec->inputs = {{v.r, m}};
    for (auto& o : rec->others)
      if (o.is_reg()) {
        int u = regid(P, o);
        rec->inputs.push_back({u, w.rd(u, m)});
      }
    return true;
  }

  std::vector<int> required() const {
    std::set<int> req;
    if (flags & F_PRUNE) {
      for (int r = 0; r < P.nregs(); r++)
        if (L.in[c][r]) req.insert(idx.at({r, w.rd(r, c)}));
    } else {
      for (int j = p; j < c; j++)
        if (w.liveout_def(j)) req.insert(idx.at({P.ins[j].defreg, j}));
      for (int r = 0; r < P.nregs(); r++)
        if (L.in[c][r] && w.rd(r, c) == PRE) req.insert(idx.at({r, PRE}));
    }
    return {req.begin(), req.end()};
  }

  // Values obtainable at preempt with their first derivation (passes in value order).
  void preempt_derivations() {
    der.assign(U.size(), {});
    for (size_t i = 0; i < U.size(); i++)
      if (w.is_current(U[i])) der[i] = {SK::C, -1, true};
    for (int m : backups) {
      int s = P.ins[m].defreg;
      int i = idx.at({s, w.rd(s, m)});
      if (!der[i].present) der[i] = {SK::B, m, true};
    }
    bool changed = true;
    while (changed) {
      changed = false;
      for (auto& R : rr) {
        if (der[R.out].present) continue;
        bool all = true;
        for (int x : R.in) all = all && der[x].present;
        if (all) {
          der[R.out] = {SK::R, R.j, true};
          changed = true;
        }
      }
    }
  }

  // Order-free least fixpoint (for the search): worklist over rule input counters.
  bool covers(const std::vector<char>& T0, const std::vector<int>& req) {
    known = T0;
    std::vector<int> cnt(xr.size() + rr.size());
    std::vector<int> stack;
    for (size_t k = 0; k < cnt.size(); k++) {   // counts against T0 only
      const Rule& R = k < xr.size() ? xr[k] : rr[k - xr.size()];
      int n = 0;
      for (int x : R.in) n += !T0[x];
      cnt[k] = n;
    }
    for (size_t k = 0; k < cnt.size(); k++) {
      const Rule& R = k < xr.size() ? xr[k] : rr[k - xr.size()];
      if (cnt[k] == 0 && !known[R.out]) {
        known[R.out] = 1;
        stack.push_back(R.out);
      }
    }
    while (!stack.empty()) {
      int v = stack.back();
      stack.pop_back();
      for (int k : users[v]) {
        if (--cnt[k] == 0) {
          const Rule& R = k < (int)xr.size() ? xr[k] : rr[k - xr.size()];
          if (!known[R.out]) {
            known[R.out] = 1;
            stack.push_back(R.out);
          }
        }
      }
    }
    for (int q : req)
      if (!known[q]) return false;
    return true;
  }

  std::vector<int> relevant(const std::vector<int>& req) const {
    std::vector<char> rel(U.size(), 0);
    for (int q : req) rel[q] = 1;
    bool changed = true;
    while (changed) {
      changed = false;
      for (auto* rules : {&xr, &rr})
        for (auto& R : *rules)
          if (rel[R.out])
            for (int x : R.in)
              if (!rel[x]) rel[x] = 1, changed = true;
    }
    std::vector<int> out;
    for (size_t i = 0; i < U.size(); i++)
      if (rel[i] && der[i].present) out.push_back((int)i);
    return out;
  }

  uint32_t vbytes(int i) const { return P.is_vec(U[i].r) ? VEC_B : SCA_B; }

  void dfs(size_t i, uint32_t bytes) {
    if (++nodes > cfg->budget) {
      aborted = true;
      return;
    }
    auto key = std::make_pair(bytes, (uint32_t)Tcur.size());
    if (covers(Tmask, req)) {
      if (key < best_key) {
        best_key = key;
        bestT = Tcur;
        found = true;
      }
      return;
    }
    if (i == cand.size() || aborted) return;
    if (std::make_pair(bytes + min_rest[i], (uint32_t)Tcur.size() + 1) >= best_key) return;
    std::vector<char> all = Tmask;   // can the remaining candidates still make it?
    for (size_t k = i; k < cand.size(); k++) all[cand[k]] = 1;
    if (!covers(all, req)) return;
    Tmask[cand[i]] = 1;
    Tcur.push_back(cand[i]);
    dfs(i + 1, bytes + vbytes(cand[i]));
    Tcur.pop_back();
    Tmask[cand[i]] = 0;
    if (!aborted) dfs(i + 1, bytes);
  }

  // Returns the exact plan, or an invalid plan if the search was skipped /
  // truncated (the caller then keeps the greedy plan).
  Plan solve(const Plan& greedy, ExactCfg* cfg_) {
    cfg = cfg_;
    preempt_derivations();
    req = required();
    cand = relevant(req);
    users.assign(U.size(), {});
    for (size_t k = 0; k < xr.size() + rr.size(); k++) {
      const Rule& R = k < xr.size() ? xr[k] : rr[k - xr.size()];
      for (int x : R.in) users[x].push_back((int)k);
    }
    cfg->windows++;
    // Reductions that cannot change the minimum or its tie-break: a candidate
    // without which even all the others do not suffice is in every feasible T
    // (forced; common to all solutions, so the lexicographic order of the rest
    // decides ties); a candidate derivable from the forced ones is in no
    // minimal T.
    std::vector<char> all(U.size(), 0), forced(U.size(), 0);
    for (int u : cand) all[u] = 1;
    if (!covers(all, req)) {
      if (greedy.valid) cfg->fallback++;
      return Plan{};
    }
    uint32_t fbytes = 0;
    for (int u : cand) {
      all[u] = 0;
      if (!covers(all, req)) forced[u] = 1, fbytes += vbytes(u), Tcur.push_back(u);
      all[u] = 1;
    }
    covers(forced, req);
    std::vector<int> rest;
    for (int u : cand)
      if (!forced[u] && !known[u]) rest.push_back(u);
    cand = rest;
    if (cand.size() > cfg->max_cand) {
      cfg->truncated++;
      return Plan{};
    }
    min_rest.assign(cand.size() + 1, UINT32_MAX / 2);
    for (size_t k = cand.size(); k-- > 0;) min_rest[k] = std::min(min_rest[k + 1], vbytes(cand[k]));
    // greedy's saved set is feasible here, so its key bounds the minimum
    best_key = greedy.valid ? std::make_pair(greedy.payload_bytes, (uint32_t)greedy.saved.size() + 1)
                            : std::make_pair(UINT32_MAX, UINT32_MAX);
    Tmask = forced;
    dfs(0, fbytes);
    if (aborted) {
      cfg->truncated++;
      return Plan{};
    }
    if (!found) {            // infeasible window (or, never expected, greedy's set not found)
      if (greedy.valid) cfg->fallback++;
      return Plan{};
    }
    Plan pl = build(bestT);
    if (greedy.valid && pl.payload_bytes < greedy.payload_bytes) cfg->improved++;
    return pl;
  }

  // The plan of a saved set T (same construction as oracle/exact.py).
  Plan build(const std::vector<int>& T) {
    std::map<int, Supply> ksup;          // value -> supply (first derivation)
    std::map<int, char> src;             // saved value -> 'C' | 'B' | 'P'
    for (int i : T) {
      const Deriv& d = der[i];
      src[i] = d.k == SK::C ? 'C' : d.k == SK::B ? 'B' : 'P';
      ksup[i] = {d.k, d.arg};
    }
    std::vector<Event> events;
    std::map<int, std::vector<Supply>> rx;
    std::map<int, RevertRec> rev;
    bool changed = true;
    while (changed) {
      changed = false;
      for (auto& R : xr) {
        if (rx.count(R.j) || ksup.count(R.out)) continue;
        bool all = true;
        for (int x : R.in) all = all && ksup.count(x);
        if (!all) continue;
        std::vector<Supply> s;
        for (int x : R.in) s.push_back(ksup.at(x));
        rx[R.j] = s;
        ksup[R.out] = {SK::X, R.j};
        events.push_back({true, R.j, U[R.out]});
        changed = true;
      }
      for (auto& R : rr) {
        if (ksup.count(R.out)) continue;
        bool all = true;
        for (int x : R.in) all = all && ksup.count(x);
        if (!all) continue;
        RevertRec rec = rrec.at(R.out);
        for (int x : R.in) rec.supplies.push_back(ksup.at(x));
        rev[R.out] = rec;
        ksup[R.out] = {SK::R, R.j};
        events.push_back({false, R.j, U[R.out]});
        changed = true;
      }
    }
    // demand-driven pruning from the required values (in value order)
    std::set<int> used_x, used_res, used_pre;
    std::map<int, char> S;
    std::function<void(int)> pre = [&](int v) {
      if (!used_pre.insert(v).second) return;
      const RevertRec& rec = rrec.at(v);
      for (auto& x : rec.inputs) {
        int xi = idx.at(x);
        if (der[xi].k == SK::R) pre(xi);
      }
    };
    std::function<void(int)> demand = [&](int v) {
      auto it = src.find(v);
      if (it != src.end()) {
        S[v] = it->second;
        if (it->second == 'P') pre(v);
        return;
      }
      const Supply& s = ksup.at(v);
      if (s.k == SK::X) {
        if (used_x.insert(s.arg).second)
          for (auto& x : w.opvals(s.arg)) demand(idx.at(x));
      } else if (used_res.insert(v).second) {
        for (auto& x : rev.at(v).inputs) demand(idx.at(x));
      }
    };
    for (int q : req) demand(q);
    Plan pl;
    pl.valid = true;
    pl.c = c;
    pl.p = p;
    pl.kind = 0;
    for (auto& [i, s] : S) {
      SavedVal sv{s, U[i], -1};
      if (s == 'B') sv.bkp_m = der[i].arg;
      pl.saved.push_back(sv);
      (P.is_vec(U[i].r) ? pl.n_vec : pl.n_sca)++;
      pl.payload_bytes += vbytes(i);
    }
    // at-preempt chains: inputs supplied by their preempt derivation
    std::vector<int> prev(used_pre.begin(), used_pre.end());
    std::stable_sort(prev.begin(), prev.end(), [&](int a, int b) { return rrec.at(a).m > rrec.at(b).m; });
    for (int v : prev) {
      RevertRec rec = rrec.at(v);
      for (auto& x : rec.inputs) {
        const Deriv& d = der[idx.at(x)];
        rec.supplies.push_back({d.k, d.k == SK::C ? -1 : d.arg});
      }
      pl.pre_reverts.push_back(rec);
      pl.revert_info[U[v]] = rec;
    }
    for (int v : used_res) pl.revert_info[U[v]] = rev.at(v);
    for (auto& e : events)
      if ((e.is_x && used_x.count(e.j)) || (!e.is_x && used_res.count(idx.at(e.v)))) pl.schedule.push_back(e);
    for (int j : used_x) pl.reexec_supply[j] = rx.at(j);
    for (int r = 0; r < P.nregs(); r++)
      if (L.in[c][r]) {
        int d = w.rd(r, c);
        pl.final_.push_back({r, d == PRE ? Supply{SK::C, -1} : ksup.at(idx.at({r, d}))});
      }
    pl.n_rev_pre = (uint32_t)used_pre.size();
    pl.n_rev_res = (uint32_t)used_res.size();
    pl.n_reexec = (uint32_t)used_x.size();
    return pl;
  }

  struct Rule {
    int out = -1, j = -1;
    std::vector<int> in;
  };
  const Program& P;
  const Liveness& L;
  Window w;
  int p, c;
  uint32_t flags;
  std::vector<Val> U;
  std::map<Val, int> idx;
  std::vector<int> backups;
  std::vector<Rule> xr, rr;
  std::map<int, RevertRec> rrec;
  std::map<int, int> xr_of_out;
  std::vector<Deriv> der;
  std::vector<std::vector<int>> users;
  std::vector<char> known, Tmask;
  std::vector<int> req, cand, Tcur, bestT;
  std::vector<uint32_t> min_rest;
  std::pair<uint32_t, uint32_t> best_key;
  uint64_t nodes = 0;
  bool aborted = false, found = false;
  ExactCfg* cfg = nullptr;
};

Plan window_plan(const Program& P, const Liveness& L, const DefIndex& D, int p, int c, const std::vector<int>& bk,
                 uint32_t flags, ExactCfg* ex = nullptr) {
  if (!(flags & F_RELAXED)) return basic_plan(P, L, D, p, c);
  Plan greedy;
  {
    Window w(P, L, D, p, c, (flags & F_OSRB) ? bk : std::vector<int>{}, flags);
    w.sweep();
    if ((flags & F_PRUNE) || w.feasible()) greedy = w.plan(0);
  }
  if ((flags & F_EXACT) && ex) {
    ExactWin xw(P, L, D, p, c, bk, flags);
    Plan pl = xw.solve(greedy, ex);
    if (pl.valid) return pl;
  }
  return greedy;
}

// CTXB_RANK_RESUME (NEXT N4; the paper ranks by preemption latency only and
// notes that re-execution can dominate resuming): estimated
// preempt + resume cost of a plan in context-byte units,
//   E = 2 * payload + re-executed load bytes + level_bytes * (levels - 1)
//     + instr_bytes * (#reverts + #re-executions),
// levels = memory round trips on the resume schedule: restored values at 1,
// a re-executed load at 1 + its deepest operand, other ops at their deepest.
uint64_t resume_estimate(const Program& P, const Plan& pl, uint32_t instr_bytes, uint32_t level_bytes) {
  std::set<std::pair<int, int>> saved_p;   // (reg, m) recovered at preempt and saved
  for (auto& sv : pl.saved)
    if (sv.src == 'P') saved_p.insert({sv.v.r, pl.revert_info.at(sv.v).m});
  std::map<int, int> lx;
  std::map<std::pair<int, int>, int> lr;
  auto level = [&](int reg, const Supply& s) -> int {
    switch (s.k) {
      case SK::C:
      case SK::B: return 1;
      case SK::X: return lx.at(s.arg);
      case SK::R: return saved_p.count({reg, s.arg}) ? 1 : lr.at({reg, s.arg});
    }
    return 1;
  };
  int depth = pl.saved.empty() ? 0 : 1;
  uint64_t load_bytes = 0;
  for (auto& e : pl.schedule) {
    int l = 0;
    if (e.is_x) {
      const Instr& I = P.ins[e.j];
      const std::vector<Supply>& sup = pl.reexec_supply.at(e.j);
      for (size_t k = 0; k < I.uses.size(); k++) l = std::max(l, level(I.uses[k], sup[k]));
      if (I.op == Op::Ldg) {
        l += 1;
        load_bytes += P.is_vec(I.defreg) ? VEC_B : SCA_B;
      }
      lx[e.j] = l;
    } else {
      const RevertRec& rec = pl.revert_info.at(e.v);
      for (size_t k = 0; k < rec.inputs.size(); k++) l = std::max(l, level(rec.inputs[k].r, rec.supplies[k]));
      lr[{e.v.r, rec.m}] = l;
    }
    depth = std::max(depth, l);
  }
  uint64_t ops = pl.schedule.size() + pl.pre_reverts.size();
  return 2ull * pl.payload_bytes + load_bytes + (uint64_t)level_bytes * (uint64_t)std::max(0, depth - 1) +
         (uint64_t)instr_bytes * ops;
}

Plan best_plan(const Program& P, const Liveness& L, const DefIndex& D, const std::vector<int>& heads, int c,
               const std::vector<int>& bk, uint32_t flags, uint32_t instr_bytes = 8, uint32_t level_bytes = 512,
               ExactCfg* ex = nullptr) {
  Plan best;
  std::vector<int64_t> bc;
  for (int p = c; p >= heads[c]; p--) {
    Plan pl = window_plan(P, L, D, p, c, bk, flags, ex);
    if (!pl.valid) continue;
    std::vector<int64_t> k;
    if (flags & F_RANK_RESUME) k.push_back((int64_t)resume_estimate(P, pl, instr_bytes, level_bytes));
    for (int x : pl.cost()) k.push_back(x);
    if (!best.valid || k < bc) {
      best = std::move(pl);
      bc = k;
    }
  }
  return best;
}

Plan full_plan(const Program& P, const Liveness& L, int c) {
  (void)L;
  Plan pl;
  pl.valid = true;
  pl.c = pl.p = c;
  pl.kind = 2;
  for (int r = 0; r < P.nregs(); r++) {
    pl.saved.push_back({'C', {r, PRE}, -1});
    pl.final_.push_back({r, {SK::C, -1}});
  }
  pl.n_vec = P.nv;
  pl.n_sca = P.ns;
  pl.payload_bytes = VEC_B * P.nv + SCA_B * P.ns;
  return pl;
}

// R-7: irreversible scalar defs whose old value is read in the same BB.
std::vector<int> osrb_candidates(const Program& P) {
  std::vector<int> out;
  for (auto [s, e] : P.bbs)
    for (int m = s; m < e; m++) {
      const Instr& I = P.ins[m];
      int r = I.defreg;
      if (r < 0 || P.is_vec(r)) continue;
      RevKind k;
      std::vector<Operand> oth;
      if (revert_spec(P, I, r, &k, &oth)) continue;
      bool read = std::find(I.uses.begin(), I.uses.end(), r) != I.uses.end();
      for (int j = m - 1; !read && j >= s; j--) {
        if (P.ins[j].defreg == r) break;
        if (std::find(P.ins[j].uses.begin(), P.ins[j].uses.end(), r) != P.ins[j].uses.end()) read = true;
      }
      if (read) out.push_back(m);
    }
  return out;
}

}  // namespace

std::vector<int> Plan::cost() const {
  return {(int)payload_bytes, (int)n_rev_pre, (int)(n_reexec + n_rev_res), -p};
}

// CS-Defer combined with the site's own plans: a
// preemption arriving at site k may continue to a later site k' of the same
// basic block and save there.  Estimated latency (stalls of the in-between
// instructions ignored, as in the paper):
//   E(k -> k') = bytes(plan at k') + defer_instr_bytes * (c_k' - c_k),
// k' minimises E (ties: the earliest k', i.e. no deferral first).
static std::vector<int> defer_targets(const Program& P, const Analysis& A, uint32_t instr_bytes) {
  std::vector<int> out(A.sites.size());
  for (size_t k = 0; k < A.sites.size(); k++) {
    int c = A.sites[k], bb = P.bb_of[c];
    size_t best = k;
    uint64_t best_e = UINT64_MAX;
    for (size_t q = 0; q < A.sites.size(); q++) {
      int d = A.sites[q];
      if (d < c || P.bb_of[d] != bb) continue;
      uint64_t e = (uint64_t)A.plans[q].payload_bytes + (uint64_t)instr_bytes * (uint64_t)(d - c);
      if (e < best_e) {
        best_e = e;
        best = q;
      }
    }
    out[k] = (int)best;
  }
  return out;
}

static Analysis analyze_plans(const Program& P, const Options& opt);

// Sites are independent given the backups (each evaluates its own windows),
// so the per-site searches run on host threads; every result lands in its
// own slot, so the analysis is identical for any thread count.  Threads:
// env CTXB_ANALYZE_THREADS, default min(hardware threads, 16); 1 = serial.
static unsigned analyze_threads() {
  const char* e = getenv("CTXB_ANALYZE_THREADS");
  unsigned v = e ? (unsigned)strtoul(e, nullptr, 10) : std::min(16u, std::thread::hardware_concurrency());
  return std::max(1u, std::min(v, 256u));
}

static void parallel_for(size_t n, unsigned nt, const std::function<void(size_t, unsigned)>& fn) {
  unsigned t = (unsigned)std::min<size_t>(nt, n);
  if (t <= 1) {
    for (size_t i = 0; i < n; i++) fn(i, 0);
    return;
  }
  std::atomic<size_t> next{0};
  std::vector<std::exception_ptr> err(t);
  std::vector<std::thread> th;
  for (unsigned w = 0; w < t; w++)
    th.emplace_back([&, w] {
      try {
        // last index first: later sites of a basic block have more windows
        for (size_t i; (i = next.fetch_add(1)) < n;) fn(n - 1 - i, w);
      } catch (...) {
        err[w] = std::current_exception();
        next = n;
      }
    });
  for (auto& x : th) x.join();
  for (auto& e : err)
    if (e) std::rethrow_exception(e);
}

Analysis analyze(const Program& P, const Options& opt) {
  Analysis A = analyze_plans(P, opt);
  if (opt.flags & F_DEFER) {
    A.defer = defer_targets(P, A, opt.defer_instr_bytes);
  } else {
    A.defer.resize(A.sites.size());
    for (size_t k = 0; k < A.sites.size(); k++) A.defer[k] = (int)k;
  }
  return A;
}

static Analysis analyze_plans(const Program& P, const Options& opt0) {
  Options opt = opt0;
  opt.flags &= (7u | F_PRUNE | F_RANK_RESUME | F_EXACT);
  Liveness L = liveness(P);
  DefIndex D(P);
  Analysis A;
  A.live_in = L.in;
  A.live_out = L.out;
  A.heads = region_heads(P);
  A.sites = sites_for(P, opt);
  A.full_ir_bytes = VEC_B * P.nv + SCA_B * P.ns;
  for (int c : A.sites) {
    Window w(P, L, D, c, c, {}, 0);
    A.live.push_back(w.plan(1));
  }
  if (opt.mode == 1) {
    A.plans = A.live;
    return A;
  }
  if (opt.mode == 2 || opt.mode == 3) {
    for (int c : A.sites) A.plans.push_back(full_plan(P, L, c));
    return A;
  }
  uint32_t fl = opt.flags;
  const unsigned nt = analyze_threads();
  if ((fl & F_OSRB) && (fl & F_RELAXED)) {
    // R-7 selects backups by the bytes of the greedy R-10 choice, whatever the
    // ranking or the plan search (R-19)
    uint32_t fb = fl & ~(F_RANK_RESUME | F_EXACT);
    std::vector<uint32_t> base(A.sites.size());
    parallel_for(A.sites.size(), nt, [&](size_t k, unsigned) {
      base[k] = best_plan(P, L, D, A.heads, A.sites[k], {}, fb).payload_bytes;
    });
    for (int m : osrb_candidates(P)) {
      // m is selected if it shrinks the plan of any site after it in its window
      int bbm = P.bb_of[m];
      std::vector<size_t> ks;
      for (size_t k = 0; k < A.sites.size(); k++) {
        int c = A.sites[k];
        if (c < (int)P.ins.size() && P.bb_of[c] == bbm && c > m && A.heads[c] <= m) ks.push_back(k);
      }
      std::atomic<bool> gain{false};
      parallel_for(ks.size(), nt, [&](size_t i, unsigned) {
        if (gain.load()) return;
        if (best_plan(P, L, D, A.heads, A.sites[ks[i]], {m}, fb).payload_bytes < base[ks[i]]) gain = true;
      });
      if (gain) A.backups.push_back(m);
    }
  }
  std::vector<ExactCfg> ex(nt);
  for (auto& e : ex)
    if (opt.exact_budget) e.budget = opt.exact_budget;
  A.plans.resize(A.sites.size());
  parallel_for(A.sites.size(), nt, [&](size_t k, unsigned w) {
    A.plans[k] = best_plan(P, L, D, A.heads, A.sites[k], A.backups, fl, opt.defer_instr_bytes,
                           opt.resume_level_bytes, &ex[w]);
  });
  for (auto& e : ex) {
    A.exact_windows += e.windows;
    A.exact_truncated += e.truncated;
    A.exact_improved += e.improved;
    A.exact_fallback += e.fallback;
  }
  return A;
}

// Canonical plan text (identical format to the oracle's plan_text).
std::string plan_text(const Program& P, const Plan& pl) {
  auto vs = [&](const Val& v) { return P.regname(v.r) + "@" + (v.d == PRE ? std::string("PRE") : std::to_string(v.d)); };
  auto ss = [&](const Supply& s) -> std::string {
    switch (s.k) {
      case SK::C: return "C";
      case SK::B: return "B" + std::to_string(s.arg);
      case SK::X: return "X" + std::to_string(s.arg);
      case SK::R: return "R" + std::to_string(s.arg);
    }
    return "?";
  };
  std::ostringstream o;
  o << "c=" << pl.c << " p=" << pl.p << " bytes=" << pl.payload_bytes << " nv=" << pl.n_vec << " ns=" << pl.n_sca;
  o << " save=";
  for (size_t i = 0; i < pl.saved.size(); i++) o << (i ? "," : "") << pl.saved[i].src << ":" << vs(pl.saved[i].v);
  o << " pre=";
  for (size_t i = 0; i < pl.pre_reverts.size(); i++)
    o << (i ? "," : "") << vs(pl.pre_reverts[i].v) << "/m" << pl.pre_reverts[i].m;
  o << " sched=";
  for (size_t i = 0; i < pl.schedule.size(); i++) {
    const Event& e = pl.schedule[i];
    o << (i ? "," : "");
    if (e.is_x) {
      o << "X" << e.j << "(";
      const auto& sup = pl.reexec_supply.at(e.j);
      for (size_t k = 0; k < sup.size(); k++) o << (k ? "," : "") << ss(sup[k]);
      o << ")";
    } else {
      const RevertRec& r = pl.revert_info.at(e.v);
      o << "R" << vs(e.v) << "/m" << r.m << "(";
      for (size_t k = 0; k < r.supplies.size(); k++) o << (k ? "," : "") << ss(r.supplies[k]);
      o << ")";
    }
  }
  o << " final=";
  for (size_t i = 0; i < pl.final_.size(); i++) o << (i ? "," : "") << P.regname(pl.final_[i].first) << ":" << ss(pl.final_[i].second);
  return o.str();
}

}  // namespace ctxb
