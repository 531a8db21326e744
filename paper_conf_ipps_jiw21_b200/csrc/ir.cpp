// IR v1 parser.  The IR stands in for the GPU assembly the
// paper's pass runs on (Figs 2-6 list GCN-style instructions such as
// `XOR r3, r4, 0xF`): one result per instruction (R-12), warp-uniform control
// flow, explicit buffer operands.
#include <algorithm>
#include <cctype>
#include <set>
#include <sstream>

#include "ctxb_internal.h"

namespace ctxb {
namespace {

std::string trim(const std::string& s) {
  size_t a = 0, b = s.size();
  while (a < b && std::isspace((unsigned char)s[a])) a++;
  while (b > a && std::isspace((unsigned char)s[b - 1])) b--;
  return s.substr(a, b - a);
}

[[noreturn]] void fail(int line, const std::string& msg) {
  throw ParseError("line " + std::to_string(line) + ": " + msg);
}

bool is_ident(const std::string& s) {
  if (s.empty() || !(std::isalpha((unsigned char)s[0]) || s[0] == '_')) return false;
  for (char ch : s)
    if (!(std::isalnum((unsigned char)ch) || ch == '_')) return false;
  return true;
}

bool all_digits(const std::string& s, size_t from = 0) {
  if (s.size() <= from) return false;
  for (size_t i = from; i < s.size(); i++)
    if (!std::isdigit((unsigned char)s[i])) return false;
  return true;
}

const char* kSpecials[] = {"tid", "laneid", "ntid", "ctaid", "nctaid", "warpid", "nwarps"};

struct Parser {
  Program P;
  int line = 0;

  Operand opd(const std::string& t0) {
    std::string t = trim(t0);
    Operand o;
    if (t.size() >= 2 && (t[0] == 'v' || t[0] == 's') && all_digits(t, 1)) {
      o.kind = t[0] == 'v' ? OK::V : OK::S;
      o.val = (uint32_t)std::stoul(t.substr(1));
      return o;
    }
    if (t.size() == 10 && t[0] == '0' && t[1] == 'f') {
      for (size_t i = 2; i < 10; i++)
        if (!std::isxdigit((unsigned char)t[i])) fail(line, "bad operand " + t);
      o.kind = OK::Imm;
      o.val = (uint32_t)std::stoul(t.substr(2), nullptr, 16);
      return o;
    }
    {
      bool neg = !t.empty() && t[0] == '-';
      std::string u = neg ? t.substr(1) : t;
      bool hex = u.size() > 2 && u[0] == '0' && (u[1] == 'x' || u[1] == 'X');
      bool ok = false;
      if (hex) {
        ok = true;
        for (size_t i = 2; i < u.size(); i++)
          if (!std::isxdigit((unsigned char)u[i])) ok = false;
      } else {
        ok = all_digits(u);
      }
      if (ok) {
        if (u.size() > 20) fail(line, "immediate out of range: " + t);
        unsigned long long v = std::stoull(u, nullptr, hex ? 16 : 10);
        long long sv = neg ? -(long long)v : (long long)v;
        if (sv < -(1LL << 31) || sv >= (1LL << 32) || (neg && v > (1ULL << 31)))
          fail(line, "immediate out of range: " + t);
        o.kind = OK::Imm;
        o.val = (uint32_t)(sv & 0xFFFFFFFFLL);
        return o;
      }
    }
    if (!t.empty() && t[0] == '%') {
      std::string n = t.substr(1);
      for (int i = 0; i < 7; i++)
        if (n == kSpecials[i]) {
          o.kind = OK::Sp;
          o.val = (uint32_t)i;
          return o;
        }
      for (size_t i = 0; i < P.uniforms.size(); i++)
        if (P.uniforms[i] == n) {
          o.kind = OK::Sp;
          o.val = (uint32_t)(SP_UNIFORM_BASE + i);
          return o;
        }
      fail(line, "unknown special " + t);
    }
    fail(line, "bad operand '" + t + "'");
  }

  Operand dstreg(const std::string& t) {
    Operand o = opd(t);
    if (!o.is_reg()) fail(line, "destination must be a register");
    return o;
  }

  void mem(const std::string& t0, Instr& I) {
    std::string t;
    for (char ch : t0)
      if (!std::isspace((unsigned char)ch)) t += ch;
    size_t lb = t.find('[');
    if (lb == std::string::npos || t.back() != ']') fail(line, "expected BUF[idx], got '" + t0 + "'");
    std::string b = t.substr(0, lb);
    if (!is_ident(b)) fail(line, "expected BUF[idx], got '" + t0 + "'");
    auto it = std::find(P.buf_names.begin(), P.buf_names.end(), b);
    if (it == P.buf_names.end()) fail(line, "unknown buffer " + b);
    I.buf = (int)(it - P.buf_names.begin());
    I.idx = opd(t.substr(lb + 1, t.size() - lb - 2));
  }

  static std::vector<std::string> split_ops(const std::string& rest) {
    std::vector<std::string> out;
    int depth = 0;
    std::string cur;
    for (char ch : rest) {
      if (ch == '[') depth++;
      if (ch == ']') depth--;
      if (ch == ',' && depth == 0) {
        out.push_back(trim(cur));
        cur.clear();
      } else {
        cur += ch;
      }
    }
    if (!trim(cur).empty()) out.push_back(trim(cur));
    return out;
  }

  Instr instr(std::string s) {
    Instr I;
    I.line = line;
    I.text = s;
    Operand guard;
    if (!s.empty() && s[0] == '@') {
      size_t sp = s.find_first_of(" \t");
      if (sp == std::string::npos) fail(line, "bad guard");
      guard = opd(s.substr(1, sp - 1));
      if (!guard.is_reg()) fail(line, "guard must be a register");
      s = trim(s.substr(sp));
    }
    size_t sp = s.find_first_of(" \t");
    std::string opc = sp == std::string::npos ? s : s.substr(0, sp);
    std::vector<std::string> ops = sp == std::string::npos ? std::vector<std::string>{} : split_ops(s.substr(sp));
    static const std::map<std::string, Op> alu2 = {
        {"iadd", Op::IAdd}, {"isub", Op::ISub}, {"imul", Op::IMul}, {"and", Op::And}, {"or", Op::Or},
        {"xor", Op::Xor},   {"shl", Op::Shl},   {"shr", Op::Shr},   {"sar", Op::Sar}, {"rotl", Op::RotL},
        {"rotr", Op::RotR}, {"umin", Op::UMin}, {"umax", Op::UMax}, {"imin", Op::IMin}, {"imax", Op::IMax},
        {"fadd", Op::FAdd}, {"fsub", Op::FSub}, {"fmul", Op::FMul}};
    static const std::map<std::string, Op> alu1 = {{"mov", Op::Mov}, {"not", Op::Not}, {"neg", Op::Neg},
                                                   {"i2f", Op::I2F}, {"u2f", Op::U2F}, {"f2i", Op::F2I}};
    static const std::map<std::string, Op> alu3 = {{"ffma", Op::FFma}, {"imad", Op::IMad}, {"sel", Op::Sel}};
    if (opc.rfind("setp.", 0) == 0) {
      std::vector<std::string> bits;
      std::stringstream ss(opc);
      std::string x;
      while (std::getline(ss, x, '.')) bits.push_back(x);
      static const char* cmps[] = {"eq", "ne", "lt", "le", "gt", "ge"};
      static const char* tys[] = {"u", "s", "f"};
      int ci = -1, ti = -1;
      if (bits.size() == 3) {
        for (int i = 0; i < 6; i++)
          if (bits[1] == cmps[i]) ci = i;
        for (int i = 0; i < 3; i++)
          if (bits[2] == tys[i]) ti = i;
      }
      if (ci < 0 || ti < 0 || ops.size() != 3) fail(line, "bad setp '" + s + "'");
      I.op = Op::Setp;
      I.cmp = (uint8_t)ci;
      I.cmpt = (uint8_t)ti;
      I.dst = dstreg(ops[0]);
      I.srcs = {opd(ops[1]), opd(ops[2])};
    } else if (alu2.count(opc)) {
      if (ops.size() != 3) fail(line, opc + " takes 3 operands");
      I.op = alu2.at(opc);
      I.dst = dstreg(ops[0]);
      I.srcs = {opd(ops[1]), opd(ops[2])};
    } else if (alu1.count(opc)) {
      if (ops.size() != 2) fail(line, opc + " takes 2 operands");
      I.op = alu1.at(opc);
      I.dst = dstreg(ops[0]);
      I.srcs = {opd(ops[1])};
    } else if (alu3.count(opc)) {
      if (ops.size() != 4) fail(line, opc + " takes 4 operands");
      I.op = alu3.at(opc);
      I.dst = dstreg(ops[0]);
      I.srcs = {opd(ops[1]), opd(ops[2]), opd(ops[3])};
    } else if (opc == "ldg") {
      if (ops.size() != 2) fail(line, "ldg d, BUF[idx]");
      I.op = Op::Ldg;
      mem(ops[1], I);
      I.dst = dstreg(ops[0]);
    } else if (opc == "stg") {
      if (ops.size() != 2) fail(line, "stg BUF[idx], a");
      I.op = Op::Stg;
      mem(ops[0], I);
      I.srcs = {opd(ops[1])};
    } else if (opc == "atom.add" || opc == "atom.cas") {
      size_t n = opc == "atom.add" ? 3 : 4;
      if (ops.size() != n) fail(line, "bad " + opc);
      I.op = opc == "atom.add" ? Op::AtomAdd : Op::AtomCas;
      if (ops[0] != "_") I.dst = dstreg(ops[0]);
      mem(ops[1], I);
      for (size_t k = 2; k < n; k++) I.srcs.push_back(opd(ops[k]));
    } else if (opc == "bra") {
      if (ops.size() != 1) fail(line, "bra LABEL");
      I.op = Op::Bra;
      I.target = ops[0];
    } else if (opc == "brnz" || opc == "brz") {
      if (ops.size() != 2) fail(line, opc + " s, LABEL");
      I.op = opc == "brnz" ? Op::Brnz : Op::Brz;
      I.srcs = {opd(ops[0])};
      I.target = ops[1];
    } else if (opc == "exit") {
      if (!ops.empty()) fail(line, "exit takes no operands");
      I.op = Op::Exit;
    } else if (opc == "bar") {
      if (!ops.empty()) fail(line, "bar takes no operands");
      I.op = Op::Bar;
    } else if (opc == "lds") {
      if (ops.size() != 2) fail(line, "lds d, idx");
      I.op = Op::Lds;
      I.dst = dstreg(ops[0]);
      I.idx = opd(ops[1]);
    } else if (opc == "sts") {
      if (ops.size() != 2) fail(line, "sts idx, a");
      I.op = Op::Sts;
      I.idx = opd(ops[0]);
      I.srcs = {opd(ops[1])};
    } else {
      fail(line, "unknown opcode '" + opc + "'");
    }
    if (guard.kind != OK::None && !(I.op == Op::Ldg || I.op == Op::Stg || I.op == Op::AtomAdd || I.op == Op::AtomCas ||
                                    I.op == Op::Lds || I.op == Op::Sts))
      fail(line, "guards only on memory ops");
    I.guard = guard;
    return I;
  }

  void run(const std::string& text) {
    bool have_name = false, have_nv = false, have_ns = false, have_block = false;
    std::vector<std::pair<int, std::string>> body;
    std::stringstream ss(text);
    std::string raw;
    int ln = 0;
    while (std::getline(ss, raw)) {
      ln++;
      line = ln;
      size_t h = raw.find('#');
      std::string s = trim(h == std::string::npos ? raw : raw.substr(0, h));
      if (s.empty()) continue;
      if (s[0] == '.') {
        std::vector<std::string> parts;
        std::stringstream ps(s);
        std::string w;
        while (ps >> w) parts.push_back(w);
        const std::string& d = parts[0];
        auto reserved = [&](const std::string& n) {
          for (auto* sp : kSpecials)
            if (n == sp) return true;
          return std::find(P.uniforms.begin(), P.uniforms.end(), n) != P.uniforms.end();
        };
        if (d == ".kernel" && parts.size() == 2) {
          P.name = parts[1];
          have_name = true;
        } else if (d == ".buffer" && parts.size() == 3 && (parts[1] == "ro" || parts[1] == "rw" || parts[1] == "wo")) {
          if (std::find(P.buf_names.begin(), P.buf_names.end(), parts[2]) != P.buf_names.end())
            fail(ln, "duplicate buffer " + parts[2]);
          if (!is_ident(parts[2])) fail(ln, "bad buffer name");
          P.buf_names.push_back(parts[2]);
          P.buf_kinds.push_back(parts[1] == "ro" ? B_RO : parts[1] == "rw" ? B_RW : B_WO);
        } else if (d == ".uniform" && parts.size() == 2) {
          if (reserved(parts[1]) || !is_ident(parts[1])) fail(ln, "bad uniform name " + parts[1]);
          P.uniforms.push_back(parts[1]);
        } else if (d == ".smem" && parts.size() == 2 && all_digits(parts[1])) {
          if (parts[1].size() > 6 || std::stoi(parts[1]) > 12288) fail(ln, ".smem too large (max 12288 words)");
          P.smem = std::stoi(parts[1]);
        } else if ((d == ".vregs" || d == ".sregs" || d == ".block") && parts.size() == 2 && all_digits(parts[1])) {
          if (parts[1].size() > 6) fail(ln, "value too large");
          int v = std::stoi(parts[1]);
          if (d == ".vregs") {
            P.nv = v;
            have_nv = true;
          } else if (d == ".sregs") {
            P.ns = v;
            have_ns = true;
          } else {
            P.block = v;
            have_block = true;
          }
        } else {
          fail(ln, "bad directive '" + s + "'");
        }
        continue;
      }
      body.emplace_back(ln, s);
    }
    if (!have_name || !have_nv || !have_ns || !have_block)
      throw ParseError("missing .kernel/.vregs/.sregs/.block");
    if (P.block <= 0 || P.block % 32 || P.block > 1024)
      throw ParseError(".block must be a positive multiple of 32, <= 1024");
    if (P.nv > 4096 || P.ns > 4096) throw ParseError("too many registers");

    std::map<std::string, int> label_at;
    bool poll_pending = false;
    for (auto& [l, s] : body) {
      line = l;
      if (s.back() == ':' && is_ident(s.substr(0, s.size() - 1))) {
        std::string lab = s.substr(0, s.size() - 1);
        if (label_at.count(lab)) fail(l, "duplicate label " + lab);
        label_at[lab] = (int)P.ins.size();
        continue;
      }
      if (s == "poll") {
        poll_pending = true;
        continue;
      }
      Instr I = instr(s);
      if (poll_pending) {
        P.explicit_sites.push_back((int)P.ins.size());
        poll_pending = false;
      }
      P.ins.push_back(std::move(I));
    }
    if (poll_pending) throw ParseError("'poll' after the last instruction");
    if (P.ins.empty()) throw ParseError("empty kernel");
    int n = (int)P.ins.size();
    std::set<int> leaders = {0};
    for (auto& [lab, i] : label_at) {
      if (i >= n) throw ParseError("label " + lab + " at end of kernel");
      leaders.insert(i);
    }
    for (int i = 0; i < n; i++) {
      Op o = P.ins[i].op;
      if ((o == Op::Bra || o == Op::Brnz || o == Op::Brz || o == Op::Exit) && i + 1 < n) leaders.insert(i + 1);
    }
    std::vector<int> ls(leaders.begin(), leaders.end());
    P.bb_of.assign(n, 0);
    std::map<int, int> start_to_bb;
    for (size_t k = 0; k < ls.size(); k++) {
      int s0 = ls[k], e0 = k + 1 < ls.size() ? ls[k + 1] : n;
      P.bbs.emplace_back(s0, e0);
      start_to_bb[s0] = (int)k;
      for (int i = s0; i < e0; i++) P.bb_of[i] = (int)k;
    }
    for (auto& [lab, i] : label_at) P.labels[lab] = start_to_bb[i];
    if (!(P.ins.back().op == Op::Bra || P.ins.back().op == Op::Exit))
      throw ParseError("the last instruction must be 'bra' or 'exit'");
    P.succ.resize(P.bbs.size());
    for (size_t b = 0; b < P.bbs.size(); b++) {
      Instr& last = P.ins[P.bbs[b].second - 1];
      std::set<int> out;
      if (last.op == Op::Bra || last.op == Op::Brnz || last.op == Op::Brz) {
        if (!P.labels.count(last.target)) fail(last.line, "unknown label " + last.target);
        last.target_bb = P.labels[last.target];
        if (last.op != Op::Bra) out.insert((int)b + 1);
        out.insert(last.target_bb);
      } else if (last.op != Op::Exit) {
        out.insert((int)b + 1);
      }
      P.succ[b].assign(out.begin(), out.end());
    }
    for (auto& I : P.ins) validate(I);
    bool uses_smem = false;
    for (auto& I : P.ins) {
      P.has_barriers = P.has_barriers || I.op == Op::Bar;
      uses_smem = uses_smem || I.op == Op::Lds || I.op == Op::Sts;
    }
    if (uses_smem && !P.has_barriers)
      throw ParseError("kernels using shared memory must synchronise with 'bar' (their preemption is block-uniform at barriers)");
    if (P.has_barriers)
      for (int c : P.explicit_sites)
        if (P.ins[c].op != Op::Bar)
          fail(P.ins[c].line, "in a kernel with barriers, 'poll' may only precede 'bar' (preemption is block-uniform at barriers)");
  }

  int regid(const Operand& o) const { return o.kind == OK::V ? (int)o.val : P.nv + (int)o.val; }

  void validate(Instr& I) {
    line = I.line;
    auto chk = [&](const Operand& o) {
      if (o.kind == OK::V && (int)o.val >= P.nv) fail(line, "v" + std::to_string(o.val) + " not declared");
      if (o.kind == OK::S && (int)o.val >= P.ns) fail(line, "s" + std::to_string(o.val) + " not declared");
    };
    for (auto& o : I.srcs) chk(o);
    chk(I.idx);
    chk(I.guard);
    chk(I.dst);
    if (I.dst.kind == OK::S) {
      bool ok = true;
      for (auto& o : I.srcs) ok = ok && o.uniform();
      if (I.idx.kind != OK::None) ok = ok && I.idx.uniform();
      if (I.guard.kind != OK::None) ok = ok && I.guard.uniform();
      if (!ok) fail(line, "scalar destination needs uniform operands");
    }
    if ((I.op == Op::Brnz || I.op == Op::Brz) && I.srcs[0].kind != OK::S)
      fail(line, "branch condition must be a scalar register");
    if ((I.op == Op::Lds || I.op == Op::Sts) && P.smem == 0) fail(line, std::string(I.op == Op::Lds ? "lds" : "sts") + " needs a .smem declaration");
    if (I.op == Op::Lds || I.op == Op::Sts || I.op == Op::Bar) {
      I.defreg = I.dst.is_reg() ? regid(I.dst) : -1;
      I.uses.clear();
      for (auto& o : I.srcs)
        if (o.is_reg()) I.uses.push_back(regid(o));
      if (I.idx.is_reg()) I.uses.push_back(regid(I.idx));
      if (I.guard.is_reg()) I.uses.push_back(regid(I.guard));
      return;
    }
    if (I.op == Op::Ldg && P.buf_kinds[I.buf] == B_WO) fail(line, "load from write-only buffer " + P.buf_names[I.buf]);
    if ((I.op == Op::Stg || I.op == Op::AtomAdd || I.op == Op::AtomCas) && P.buf_kinds[I.buf] == B_RO)
      fail(line, "write to read-only buffer " + P.buf_names[I.buf]);
    if ((I.op == Op::AtomAdd || I.op == Op::AtomCas) && P.buf_kinds[I.buf] != B_RW)
      fail(line, "atomics need an rw buffer");
    I.defreg = I.dst.is_reg() ? regid(I.dst) : -1;
    I.uses.clear();
    for (auto& o : I.srcs)
      if (o.is_reg()) I.uses.push_back(regid(o));
    if (I.idx.is_reg()) I.uses.push_back(regid(I.idx));
    if (I.guard.is_reg()) I.uses.push_back(regid(I.guard));
  }
};

}  // namespace

Program parse_ir(const std::string& text) {
  Parser p;
  p.run(text);
  return std::move(p.P);
}

}  // namespace ctxb
