// Internal data structures of libctxb (not part of the ABI).
// Written from DESIGN.md ("IR v1", "Normative reading CTXB-R1"); shares no code
// with the Python oracle under oracle/.
#pragma once
#include <cstdint>
#include <map>
#include <stdexcept>
#include <string>
#include <vector>

namespace ctxb {

struct ParseError : std::runtime_error {
  using std::runtime_error::runtime_error;
};

// ---- IR ---------------------------------------------------------------------
enum class OK : uint8_t { None, V, S, Imm, Sp };  // operand kinds

// specials: per-lane (tid, laneid) or uniform (ntid, ctaid, nctaid, warpid, nwarps, uniform params)
enum Special : int { SP_TID = 0, SP_LANEID, SP_NTID, SP_CTAID, SP_NCTAID, SP_WARPID, SP_NWARPS,
                     SP_UNIFORM_BASE = 100 };

struct Operand {
  OK kind = OK::None;
  uint32_t val = 0;  // reg index / imm bits / special id
  bool is_reg() const { return kind == OK::V || kind == OK::S; }
  bool uniform() const {
    return kind == OK::S || kind == OK::Imm || (kind == OK::Sp && val != SP_TID && val != SP_LANEID);
  }
};

enum class Op : uint8_t {
  Mov, Not, Neg, I2F, U2F, F2I,
  IAdd, ISub, IMul, And, Or, Xor, Shl, Shr, Sar, RotL, RotR, UMin, UMax, IMin, IMax,
  FAdd, FSub, FMul,
  FFma, IMad, Sel, Setp,
  Ldg, Stg, AtomAdd, AtomCas,
  Lds, Sts, Bar,              // shared memory (per block) and the block barrier (N2)
  Bra, Brnz, Brz, Exit
};

enum Cmp : uint8_t { C_EQ, C_NE, C_LT, C_LE, C_GT, C_GE };
enum CmpT : uint8_t { T_U, T_S, T_F };

struct Instr {
  Op op{};
  Operand dst;                 // kind None if no result
  std::vector<Operand> srcs;   // value operands
  int buf = -1;                // memory buffer index
  Operand idx;                 // memory index
  Operand guard;               // lane guard (kind None if absent)
  int target_bb = -1;          // branch target BB
  std::string target;          // label text
  uint8_t cmp = 0, cmpt = 0;   // setp modifiers
  int line = 0;
  std::string text;
  // register ids: vectors 0..nv-1, scalars nv..nv+ns-1 ; -1 = none
  int defreg = -1;
  std::vector<int> uses;       // in operand order: srcs, idx, guard
};

enum BufKind : uint8_t { B_RO, B_RW, B_WO };

struct Program {
  std::string name;
  std::vector<std::string> buf_names;
  std::vector<BufKind> buf_kinds;
  std::vector<std::string> uniforms;
  int nv = 0, ns = 0, block = 0;
  std::vector<Instr> ins;
  std::vector<std::pair<int, int>> bbs;   // [start, end)
  std::vector<int> bb_of;                 // per instruction
  std::vector<std::vector<int>> succ;     // per BB
  std::map<std::string, int> labels;      // label -> BB
  std::vector<int> explicit_sites;
  int smem = 0;                           // u32 words of shared memory per block
  bool has_barriers = false;
  int nregs() const { return nv + ns; }
  bool is_vec(int r) const { return r < nv; }
  std::string regname(int r) const {
    return r < nv ? "v" + std::to_string(r) : "s" + std::to_string(r - nv);
  }
};

Program parse_ir(const std::string& text);

// ---- analysis ---------------------------------------------------------------
constexpr int PRE = -1;  // value "defined before the window"

// Preemption-flag replicas (runtime + generated code): warps poll replica
// (global warp id % FLAG_REPLICAS), one per FLAG_STRIDE bytes, after the
// master word and the gather words of the flag buffer.
constexpr uint32_t FLAG_REPLICAS = 64;
constexpr uint32_t FLAG_STRIDE = 4096;

struct Val {         // (register, defining instruction or PRE)
  int r = -1;
  int d = PRE;
  bool operator<(const Val& o) const { return r != o.r ? r < o.r : d < o.d; }
  bool operator==(const Val& o) const { return r == o.r && d == o.d; }
};

enum class SK : uint8_t { C, B, X, R };  // supply kinds: CURRENT, BACKUP(m), REEXEC(j), REVERT(m)
struct Supply {
  SK k = SK::C;
  int arg = -1;
};

enum RevKind : uint8_t { RV_SUB_D, RV_ADD_D, RV_RSUB_D, RV_XOR_D, RV_NOT_D, RV_NEG_D, RV_MULINV,
                         RV_ROTR, RV_ROTL };

struct RevertRec {
  Val v;                 // recovered value
  int m = -1;            // the reverted instruction
  RevKind kind{};
  std::vector<Val> inputs;        // (r, m), then other register operands of m
  std::vector<Supply> supplies;
  std::vector<Operand> others;    // non-shared operands of m (regs, imm, specials), in order
};

struct SavedVal {
  char src;   // 'C' register at preempt, 'P' recovered at preempt, 'B' OSRB backup
  Val v;
  int bkp_m = -1;
};

struct Event {   // resume schedule entry
  bool is_x;     // true: re-execute instruction j ; false: revert (index into reverts)
  int j;
  Val v;
};

struct Plan {
  int c = 0, p = 0;
  int kind = 0;  // 0 ctxback, 1 live, 2 full, 3 basic
  std::vector<SavedVal> saved;             // sorted (vectors first, reg, d, src)
  std::vector<RevertRec> pre_reverts;      // at preempt, decreasing m
  std::vector<Event> schedule;             // resume, established order
  std::map<int, std::vector<Supply>> reexec_supply;  // j -> supplies per use
  std::map<Val, RevertRec> revert_info;    // every established revert
  std::vector<std::pair<int, Supply>> final_;   // r in LIVE_IN(c) -> supply of (r, rd(r,c))
  uint32_t payload_bytes = 0, n_vec = 0, n_sca = 0, n_rev_pre = 0, n_rev_res = 0, n_reexec = 0;
  bool valid = false;
  std::vector<int> cost() const;
};

struct Options {
  uint32_t flags = 7, mode = 0, policy = 0, every = 8, debug = 0, flag_depth = 1, min_blocks = 0;
  uint32_t defer_instr_bytes = 8;   // CS-Defer latency-estimate weight per deferred instruction
  uint32_t resume_level_bytes = 512;  // CTXB_RANK_RESUME weight of one dependent memory round trip
  uint32_t exact_budget = 0;          // CTXB_EXACT search nodes per window (0 = default)
  uint32_t load_every = 1;            // flag loads at every K-th poll visit (flag mode)
};

struct Analysis {
  std::vector<std::vector<uint8_t>> live_in, live_out;   // per instr, per reg (0/1)
  std::vector<int> heads;                               // h(c)
  std::vector<int> sites;
  std::vector<int> backups;                             // OSRB-selected instructions
  std::vector<Plan> plans;                              // per site (index into sites)
  std::vector<Plan> live;                               // LIVE plan per site
  std::vector<int> defer;                               // per site: index of the site it defers to
  uint32_t full_ir_bytes = 0;
  // CTXB_EXACT: windows searched, truncated (budget / size: greedy plan kept),
  // strictly improved over greedy, and greedy fallbacks (never expected)
  uint32_t exact_windows = 0, exact_truncated = 0, exact_improved = 0, exact_fallback = 0;
};

Analysis analyze(const Program& prog, const Options& opt);
std::string plan_text(const Program& prog, const Plan& pl);

// ---- code generation -------------------------------------------------------
struct CodegenInfo {
  uint32_t stride = 0;            // payload slot bytes per warp (multiple of 128)
  uint32_t max_payload = 0;
  uint32_t resume_maxnreg = 0;    // in: register cap of the resume kernel (0 = none)
  uint32_t n_save_stubs = 0;      // out: distinct preemption-routine bodies (P:317 sharing)
  uint32_t n_fp_shared = 0;       // out: sites entering a flashback-point routine at an offset
};
std::string generate_cuda(const Program& prog, const Analysis& an, const Options& opt,
                          CodegenInfo* info);

}  // namespace ctxb
