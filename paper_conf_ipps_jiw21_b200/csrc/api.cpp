// C ABI of libctxb (include/ctxb.h).  Compile-time part: P:311-317; runtime
// part: P:319-323 (preemption), P:313-315 (resume).
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <regex>

#include "../../include/ctxb.h"
#include "ctxb_internal.h"
#include "driver.h"

using namespace ctxb;

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

double now_ms() {
  using namespace std::chrono;
  return duration<double, std::milli>(steady_clock::now().time_since_epoch()).count();
}

struct Mod {
  CUmodule mod = nullptr;
  CUfunction run = nullptr, resume = nullptr;
};

std::string cu_err(CUresult r) {
  const char* s = nullptr;
  if (driver().ok) driver().cuGetErrorString(r, &s);
  return s ? s : ("CUresult " + std::to_string((int)r));
}

#define CU(call)                                                               \
  do {                                                                         \
    CUresult _r = (call);                                                      \
    if (_r != CUDA_SUCCESS) return fail(CTXB_E_CUDA, std::string(#call) + ": " + cu_err(_r)); \
  } while (0)

}  // namespace

struct ctxb_program {
  Program prog;
  Analysis an;
  Options opt;
  CodegenInfo cg;
  std::string src, log;
  std::vector<char> cubin;
  uint32_t num_regs = 0, regs_resume = 0;
  uint32_t poll_loop = 0;   // IR instructions on the shortest loop through a poll site (0: none)
  uint32_t spill_st = 0, spill_ld = 0, spill_st_res = 0, spill_ld_res = 0;   // ptxas -v bytes
  double t_an = 0, t_cg = 0, t_cc = 0;
  std::mutex mu;
  std::map<CUcontext, Mod> mods;
  std::map<CUcontext, uint64_t> gather_resident;   // per context: blocks a gathered resume may wait for
  struct Res {
    CUdeviceptr flag = 0, stamps = 0, forced = 0;
    uint32_t n_warps = 0;
    CUevent ev0 = nullptr, ev1 = nullptr, evf = nullptr;
    void* hflag = nullptr;    // CTXB_HOST_SIGNAL / CTXB_ARMED_SIGNAL: mapped pinned host words (else NULL)
    CUdeviceptr hflag_dev = 0;
    CUstream arm = nullptr;   // CTXB_ARMED_SIGNAL: the library's signal stream
    uint32_t gate_seq = 0;
    void* hdr_pin = nullptr;  // pinned staging for the header read-back
    uint64_t rep_off = 0;     // offset of the flag replicas in the flag buffer
    uint32_t sig_seq = 0;     // last signal value used on this flag buffer
    uint32_t drain_total = 0; // warps counted out on this flag buffer so far (mod 2^32)
  };
  std::vector<Res> pool;   // per-run device resources, reused (flags hold stale signal values only)
  int live_runs = 0;        // runs that still reference this program
  bool destroy_pending = false;   // ctxb_program_destroy came first: the last run frees it
  uint32_t full_ir_words128() const {  // 128-B rows occupied by the FULL_IR layout
    return (uint32_t)prog.nv + ((uint32_t)prog.ns * 4 + 127) / 128;
  }
  uint32_t pad_regs() const {
    if (opt.mode != CTXB_MODE_FULL_HW) return 0;
    uint32_t w = full_ir_words128();
    return num_regs > w ? num_regs - w : 0;
  }
  uint32_t full_hw_bytes() const { return (full_ir_words128() + pad_regs()) * 128u; }
  uint32_t smem_slice_bytes() const {
    if (!prog.smem) return 0;
    uint32_t nw = (uint32_t)prog.block / 32;
    return 4u * (((uint32_t)prog.smem + nw - 1) / nw);
  }
  uint32_t smem_off() const {   // the warp's smem slice follows its register payload
    uint32_t s = cg.stride;
    if (opt.mode == CTXB_MODE_FULL_HW) s = std::max(s, full_hw_bytes());
    return ((s + 127) / 128) * 128;
  }
  uint32_t stride() const {
    uint32_t s = smem_off() + ((smem_slice_bytes() + 127) / 128) * 128;
    return std::max<uint32_t>(128, s);
  }
};

// RUN_DRAINED: ctxb_preempt without stats returned as soon as the launch
// drained; the headers are read (-> PREEMPTED / DONE) on the next call that
// needs them (settle()).
enum { RUN_RUNNING = 0, RUN_PREEMPTED = 1, RUN_DONE = 2, RUN_DRAINED = 3 };

void free_program(ctxb_program* p);

struct ctxb_run {
  ctxb_program* prog = nullptr;
  CUcontext ctx = nullptr;
  Mod mod;
  uint32_t grid = 0, n_warps = 0;
  std::vector<uint64_t> bufs;
  std::vector<uint32_t> uni;
  CUdeviceptr cbuf = 0;
  uint64_t cbytes = 0, pay_off = 0, stride = 0;
  CUstream stream = nullptr;
  CUdeviceptr flag = 0, stamps = 0, forced = 0;
  void* hflag = nullptr;    // mapped pinned host words: [0] CTXB_HOST_SIGNAL word, [16] CTXB_ARMED_SIGNAL gate
  CUdeviceptr hflag_dev = 0;
  CUstream arm = nullptr;   // CTXB_ARMED_SIGNAL: stream holding the pre-enqueued signal
  uint32_t gate_seq = 0;    //   gate value that releases the armed signal of the current launch
  bool armed = false;       //   an armed signal is pending on `arm`
  bool watching = false;    // CTXB_WATCHER: the current launch's watcher warp waits for the host word
  CUdeviceptr stamps_watch = 0;   //   where the watcher stamps when it raised the flag (stamps + 32 n_warps)
  uint32_t epoch = 0;
  uint32_t rb_target = 0;   // CTXB_GATHER_RESUME: blocks with preempted warps the resume launch waits for
  int state = RUN_RUNNING;
  std::vector<uint32_t> hdr_prev, hdr;  // host header snapshots (launch e-1, e)
  bool resumed_launch = false;
  CUevent ev0 = nullptr, ev1 = nullptr;   // recorded around each launch on the run's stream
  CUevent evf = nullptr;                  // recorded on the control stream before the flag write
  void* hdr_pin = nullptr;                // pinned staging buffer for the headers (n_warps x 16 B)
  uint64_t rep_off = 0;                   // flag replicas: r->flag + rep_off + k * FLAG_STRIDE
  uint32_t sig = 0, sig_seq = 0;          // signal value of the current launch; last value used on this buffer
  uint32_t drain_base = 0, drain_total = 0;   // exit count before this launch; after it
  // CTXB_ARMED_SIGNAL: release a pending armed signal of a launch that was not
  // preempted and clear the flag it raises (off the preemption path).
  // CTXB_WATCHER: the launch will not be preempted any more (the caller waits
  // for its end, or it ended) -> the watcher exits without raising the flag.
  // Done *before* waiting for the victim: under tools that serialise kernels
  // (compute-sanitizer, ncu) the victim only starts once the watcher ends.
  void release_watcher() {
    if (!watching) return;
    watching = false;
    *(static_cast<volatile uint32_t*>(hflag) + 8) = gate_seq | 0x80000000u;
    std::atomic_thread_fence(std::memory_order_seq_cst);
  }
  void disarm() {
    if (watching) {   // the launch ended unpreempted
      release_watcher();
      driver().cuStreamSynchronize(arm);
    }
    if (!armed) return;
    armed = false;
    Driver& d = driver();
    *(static_cast<volatile uint32_t*>(hflag) + 16) = gate_seq;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    d.cuStreamSynchronize(arm);   // the armed ops ran (their value is stale now)
  }
  ~ctxb_run() {
    if (!prog) return;
    bool last = false;
    {
      std::lock_guard<std::mutex> g(prog->mu);
      if (flag) {   // return the resources to the program's pool
        // a launch still running keeps its flag / stamps: let it finish first
        // (disarming would otherwise preempt it)
        release_watcher();
        if (state == RUN_RUNNING) driver().cuStreamSynchronize(stream);
        disarm();
        prog->pool.push_back({flag, stamps, forced, n_warps, ev0, ev1, evf, hflag, hflag_dev, arm, gate_seq,
                              hdr_pin, rep_off, sig_seq, drain_total});
      }
      last = --prog->live_runs == 0 && prog->destroy_pending;
    }
    if (last) free_program(prog);   // the program was destroyed while this run lived
  }
};

namespace {

int ensure_ctx(CUcontext* out) {
  Driver& d = driver();
  if (!d.ok) return fail(CTXB_E_CUDA, d.err);
  CUcontext c = nullptr;
  CU(d.cuCtxGetCurrent(&c));
  if (!c) {
    CUdevice dev;
    CU(d.cuDeviceGet(&dev, 0));
    CU(d.cuDevicePrimaryCtxRetain(&c, dev));
    CU(d.cuCtxSetCurrent(c));
  }
  *out = c;
  return CTXB_OK;
}

int ensure_module(ctxb_program* p, CUcontext c, Mod* out) {
  if (p->cubin.empty()) return fail(CTXB_E_STATE, "program was analysed with CTXB_DEBUG_NO_COMPILE");
  std::lock_guard<std::mutex> g(p->mu);
  auto it = p->mods.find(c);
  if (it != p->mods.end()) {
    *out = it->second;
    return CTXB_OK;
  }
  Driver& d = driver();
  Mod m;
  CU(d.cuModuleLoadData(&m.mod, p->cubin.data()));
  CU(d.cuModuleGetFunction(&m.run, m.mod, "ctxb_run"));
  CU(d.cuModuleGetFunction(&m.resume, m.mod, "ctxb_resume"));
  int nr = 0;
  CU(d.cuFuncGetAttribute(&nr, CU_FUNC_ATTRIBUTE_NUM_REGS, m.run));
  if (p->num_regs == 0) p->num_regs = (uint32_t)nr;
  p->mods[c] = m;
  *out = m;
  return CTXB_OK;
}

// Register count of kernel `fn` from the cubin itself: the EIATTR_REGCOUNT
// attribute (0x2f, EIFMT_SVAL payload {u32 symbol index, u32 count}) of the
// ELF's ".nv.info" section, the symbol named through .symtab/.strtab.  (The
// ptxas -v text in the NVRTC log is not always there: it is missing when the
// process runs under ncu.)  Returns 0 if absent or malformed.
uint32_t cubin_regcount(const std::vector<char>& cb, const char* fn) {
  auto rd = [&](size_t o, size_t n, void* out) {
    if (o + n > cb.size()) return false;
    memcpy(out, cb.data() + o, n);
    return true;
  };
  uint64_t shoff = 0;
  uint16_t shent = 0, shnum = 0, shstr = 0;
  if (cb.size() < 64 || memcmp(cb.data(), "\x7f" "ELF", 4) != 0 || !rd(0x28, 8, &shoff) || !rd(0x3A, 2, &shent) ||
      !rd(0x3C, 2, &shnum) || !rd(0x3E, 2, &shstr) || shent < 64 || shstr >= shnum)
    return 0;
  struct Sec { uint32_t name = 0; uint64_t off = 0, size = 0; uint32_t link = 0; };
  std::vector<Sec> s(shnum);
  for (uint32_t i = 0; i < shnum; i++) {
    size_t o = shoff + (size_t)i * shent;
    if (!rd(o, 4, &s[i].name) || !rd(o + 0x18, 8, &s[i].off) || !rd(o + 0x20, 8, &s[i].size) ||
        !rd(o + 0x28, 4, &s[i].link))
      return 0;
  }
  auto str = [&](uint64_t base, uint32_t o) -> std::string {
    std::string out;
    for (size_t i = base + o; i < cb.size() && cb[i]; i++) out += cb[i];
    return out;
  };
  int info = -1, sym = -1;
  for (uint32_t i = 0; i < shnum; i++) {
    std::string nm = str(s[shstr].off, s[i].name);
    if (nm == ".nv.info") info = (int)i;
    if (nm == ".symtab") sym = (int)i;
  }
  if (info < 0 || sym < 0 || s[sym].link >= shnum) return 0;
  const Sec& st = s[s[sym].link];
  for (uint64_t i = s[info].off, end = s[info].off + s[info].size; i + 4 <= end;) {
    uint8_t fmt = (uint8_t)cb[i], attr = (uint8_t)cb[i + 1];
    uint16_t sz = 0;
    if (fmt != 0x04) {   // NVAL / BVAL / HVAL: 4 bytes
      i += 4;
      continue;
    }
    if (!rd(i + 2, 2, &sz)) return 0;
    if (attr == 0x2f && sz >= 8) {
      uint32_t si = 0, cnt = 0, nmo = 0;
      if (!rd(i + 4, 4, &si) || !rd(i + 8, 4, &cnt) || !rd(s[sym].off + (uint64_t)si * 24, 4, &nmo)) return 0;
      if (str(st.off, nmo) == fn) return cnt;
    }
    i += 4 + sz;
  }
  return 0;
}

int nvrtc_compile(ctxb_program* p, uint32_t* regs_run, uint32_t* regs_resume) {
  Nvrtc& n = nvrtc();
  if (!n.ok) return fail(CTXB_E_NVRTC, n.err);
  void* prog = nullptr;
  int r = n.CreateProgram(&prog, p->src.c_str(), (p->prog.name + ".cu").c_str(), 0, nullptr, nullptr);
  if (r) return fail(CTXB_E_NVRTC, std::string("nvrtcCreateProgram: ") + n.GetErrorString(r));
  const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "-lineinfo", "--fmad=false",
                        "--ptxas-options=-v", "-DNDEBUG", "-diag-suppress=177,550"};
  r = n.CompileProgram(prog, (int)(sizeof(opts) / sizeof(opts[0])), opts);
  size_t ls = 0;
  n.GetProgramLogSize(prog, &ls);
  std::string log(ls, '\0');
  if (ls) n.GetProgramLog(prog, &log[0]);
  p->log = log;
  if (r) {
    n.DestroyProgram(&prog);
    return fail(CTXB_E_NVRTC, "NVRTC compilation failed: " + log.substr(0, 4000));
  }
  size_t cs = 0;
  n.GetCUBINSize(prog, &cs);
  p->cubin.resize(cs);
  n.GetCUBIN(prog, p->cubin.data());
  n.DestroyProgram(&prog);
  // ptxas -v: "Compiling entry function 'NAME'" ... "Used N registers"
  auto regs_of = [&](const char* fn) -> uint32_t {
    size_t at = log.find(std::string("'") + fn + "'");
    if (at == std::string::npos) return 0;
    std::smatch m;
    std::string tail = log.substr(at);
    if (std::regex_search(tail, m, std::regex("Used ([0-9]+) registers"))) return (uint32_t)std::stoul(m[1]);
    return 0;
  };
  // ptxas -v: "N bytes stack frame, N bytes spill stores, N bytes spill loads"
  // after the function's "Compiling entry function" line (0 when the log is absent)
  auto spill_of = [&](const char* fn, uint32_t* st, uint32_t* ld) {
    *st = *ld = 0;
    size_t at = log.find(std::string("'") + fn + "'");
    if (at == std::string::npos) return;
    std::smatch m;
    std::string tail = log.substr(at);
    if (std::regex_search(tail, m, std::regex("([0-9]+) bytes spill stores, ([0-9]+) bytes spill loads"))) {
      *st = (uint32_t)std::stoul(m[1]);
      *ld = (uint32_t)std::stoul(m[2]);
    }
  };
  spill_of("ctxb_run", &p->spill_st, &p->spill_ld);
  spill_of("ctxb_resume", &p->spill_st_res, &p->spill_ld_res);
  *regs_run = cubin_regcount(p->cubin, "ctxb_run");
  *regs_resume = cubin_regcount(p->cubin, "ctxb_resume");
  // the two sources must agree when the log has them
  uint32_t lr = regs_of("ctxb_run"), ls2 = regs_of("ctxb_resume");
  if ((lr && lr != *regs_run) || (ls2 && ls2 != *regs_resume))
    return fail(CTXB_E_NVRTC, "register counts: cubin " + std::to_string(*regs_run) + "/" +
                                  std::to_string(*regs_resume) + " vs ptxas log " + std::to_string(lr) + "/" +
                                  std::to_string(ls2));
  if (!*regs_run) *regs_run = lr;
  if (!*regs_resume) *regs_resume = ls2;
  return CTXB_OK;
}

// Resident blocks per SM allowed by the register file (64 K 32-bit registers,
// per-warp allocation in units of 256 registers, at most 64 warps / 32 blocks).
uint32_t blocks_by_regs(uint32_t regs, uint32_t block) {
  if (regs == 0) return 32;
  uint32_t warps = (block + 31) / 32;
  uint32_t per_warp = ((regs * 32 + 255) / 256) * 256;
  uint32_t b = 65536u / (per_warp * warps);
  return std::min<uint32_t>(std::min<uint32_t>(b, 64u / warps), 32u);
}

int compile(ctxb_program* p) {
  uint32_t rr = 0, rs = 0;
  int rc = nvrtc_compile(p, &rr, &rs);
  if (rc) return rc;
  uint32_t bw = blocks_by_regs(rr, p->prog.block), bs = blocks_by_regs(rs, p->prog.block);
  if (bs < bw && bw > 0) {
    // ask ptxas for the normal kernel's occupancy (__launch_bounds__ min blocks)
    p->cg.resume_maxnreg = bw;
    uint32_t nss = p->cg.n_save_stubs;
    p->src = generate_cuda(p->prog, p->an, p->opt, &p->cg);
    (void)nss;
    rc = nvrtc_compile(p, &rr, &rs);
    if (rc) return rc;
  }
  p->num_regs = rr;
  p->regs_resume = rs;
  return CTXB_OK;
}

void pack_params(const ctxb_run* r, const ctxb_program* p, std::vector<uint64_t>& blob) {
  size_t nb = std::max<size_t>(1, p->prog.buf_names.size());
  size_t nu = std::max<size_t>(1, p->prog.uniforms.size());
  size_t words = nb + 6 + (nu + 13 + 1) / 2;
  blob.assign(words, 0);
  for (size_t i = 0; i < r->bufs.size(); i++) blob[i] = r->bufs[i];
  blob[nb + 0] = r->cbuf;
  blob[nb + 1] = r->flag;
  blob[nb + 2] = r->forced;
  blob[nb + 3] = r->stamps;
  blob[nb + 4] = r->pay_off;
  blob[nb + 5] = r->hflag_dev;
  uint32_t* u = reinterpret_cast<uint32_t*>(&blob[nb + 6]);
  for (size_t i = 0; i < r->uni.size(); i++) u[i] = r->uni[i];
  u[nu + 0] = r->epoch;
  u[nu + 1] = (uint32_t)r->stride;
  u[nu + 2] = p->pad_regs();
  u[nu + 3] = p->full_hw_bytes();
  u[nu + 4] = 0;   // `zero`: opaque 0 for the timing dependency (gtimer_after)
  u[nu + 5] = p->smem_off();
  u[nu + 6] = r->resumed_launch ? r->rb_target : 0u;
  static const uint32_t gather_timeout = [] {   // ns; bounds the wait if a block is not resident
    const char* e = getenv("CTXB_GATHER_TIMEOUT_NS");
    return e ? (uint32_t)strtoul(e, nullptr, 10) : 20000u;
  }();
  u[nu + 7] = gather_timeout;
  // CTXB_HOST_SIGNAL: R host-word reads per poll interval device-wide: each
  // warp reads once every ceil(n_warps / R) of its polls
  const char* re = getenv("CTXB_HOST_RELAYS");
  uint32_t relays = re ? (uint32_t)strtoul(re, nullptr, 10) : 1u;
  relays = relays ? relays : 1u;
  u[nu + 8] = std::max<uint32_t>(1u, (r->n_warps + relays - 1) / relays);
  u[nu + 9] = (uint32_t)r->rep_off;
  u[nu + 10] = r->sig;
  u[nu + 11] = std::max<uint32_t>(1u, r->n_warps / 32u);   // master polls: ~32 per poll interval grid-wide
  u[nu + 12] = r->drain_base;
}

int upload_forced(ctxb_run* r, const uint32_t* targets) {
  Driver& d = driver();
  if (!(r->prog->opt.debug & CTXB_DEBUG_FORCED)) {
    if (targets) return fail(CTXB_E_INVALID_ARG, "forced_targets given but the program is not CTXB_DEBUG_FORCED");
    return CTXB_OK;
  }
  if (targets) {
    CU(d.cuMemcpyHtoD(r->forced, targets, (size_t)r->n_warps * 4));
  } else {
    CU(d.cuMemsetD32Async(r->forced, 0xFFFFFFFFu, r->n_warps, r->stream));
  }
  return CTXB_OK;
}

// The preemption signal: the launch's unique value r->sig written to the
// master flag word (the kernel forwards it to the replicas it polls).  Flags
// are never reset: a later launch waits for a different value.
int write_signal(ctxb_run* r, CUstream s) {
  CU(driver().cuStreamWriteValue32(s, r->flag, r->sig, 0));
  return CTXB_OK;
}

const char* kProbeSrc = R"CUDA(
typedef unsigned int u32; typedef unsigned long long u64;
static __device__ __forceinline__ u64 gt() { u64 t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
static __device__ __forceinline__ u32 ldcv(const u32* p) { u32 v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v; }
extern "C" __global__ void ctxb_probe_spin(const u32* flag, u64* out) {
  u64 t0 = gt();
  while (ldcv(flag) == 0u) { if (gt() - t0 > 20000000ull) break; }   // 20 ms timeout
  if (threadIdx.x == 0) out[1] = gt();
}
extern "C" __global__ void ctxb_probe_stamp(u64* out) { if (threadIdx.x == 0) out[0] = gt(); }
// CTXB_WATCHER: one warp, co-resident with the victim, relays a host store to
// the device flag.  It marks itself started (the victim's launch waits for
// that, so the watcher always has its slot), then polls the host word in
// mapped pinned memory with system-scope loads: seq raises the launch's signal
// value in the master flag and every replica; seq | 0x80000000 (the launch
// ended unpreempted) makes it exit.
extern "C" __global__ void ctxb_watcher(const u32* hw, u32 seq, u32* flag, unsigned long long rep_off, u32 sig,
                                        u32* started, u64* stamp, const u32* exits, u32 exit_base, u32 nblocks) {
  const u32 lane = threadIdx.x;
  if (lane == 0) asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(started), "r"(seq) : "memory");
  // The host word only moves forward (31-bit sequence numbers, bit 31 = the
  // launch ended unpreempted): wait while it is behind seq; raise the flags
  // only for exactly seq; any later value (a newer launch's) just ends this
  // watcher, so a stale watcher can never hold the stream.  The watcher also
  // ends once every block of its launch has exited (the launch's exit count,
  // kept in device memory by the victim): an operation that waits for the
  // device to go idle (a module load, cudaFree) then waits only for the
  // victim, as it would without a watcher.
  u32 v;
  for (;;) {
    asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(hw) : "memory");
    if ((int)(((v & 0x7FFFFFFFu) - seq) << 1) >= 0) break;
    u32 e;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(e) : "l"(exits) : "memory");
    if (e - exit_base >= nblocks) return;
  }
  if (v != seq) return;
  for (u32 k = lane; k <= 64u; k += 32u) {
    u32* a = k == 0u ? flag : flag + (rep_off + (u64)(k - 1u) * 4096u) / 4u;
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(a), "r"(sig) : "memory");
  }
  if (lane == 0) *stamp = gt();
}
)CUDA";

struct Probe {
  CUmodule mod = nullptr;
  CUfunction spin = nullptr, stamp = nullptr, watch = nullptr;
};

std::mutex probe_mu;

// The probe module of context c (compiled once with NVRTC); caller holds probe_mu.
int probe_module(CUcontext c, Probe** out) {
  static std::map<CUcontext, Probe> probes;
  Probe& P = probes[c];
  Driver& d = driver();
  if (!P.mod) {
    Nvrtc& n = nvrtc();
    if (!n.ok) return fail(CTXB_E_NVRTC, n.err);
    void* prog = nullptr;
    if (n.CreateProgram(&prog, kProbeSrc, "probe.cu", 0, nullptr, nullptr)) return fail(CTXB_E_NVRTC, "probe");
    const char* opts[] = {"--gpu-architecture=sm_100a"};
    if (n.CompileProgram(prog, 1, opts)) {
      n.DestroyProgram(&prog);
      return fail(CTXB_E_NVRTC, "probe compile");
    }
    size_t cs = 0;
    n.GetCUBINSize(prog, &cs);
    std::vector<char> cubin(cs);
    n.GetCUBIN(prog, cubin.data());
    n.DestroyProgram(&prog);
    CU(d.cuModuleLoadData(&P.mod, cubin.data()));
    CU(d.cuModuleGetFunction(&P.spin, P.mod, "ctxb_probe_spin"));
    CU(d.cuModuleGetFunction(&P.stamp, P.mod, "ctxb_probe_stamp"));
    CU(d.cuModuleGetFunction(&P.watch, P.mod, "ctxb_watcher"));
  }
  *out = &P;
  return CTXB_OK;
}

// CTXB_WATCHER: launch the watcher warp of run r's current launch on the
// library's signal stream and make the victim's stream wait until it runs.
// Under Nsight Compute every kernel launch is profiled to completion inside
// the launch call, so a watcher kernel (which ends only when the host tells it
// to) would never return: no watcher there (ncu sets
// NV_COMPUTE_PROFILER_PERFWORKS_DIR); CTXB_NO_WATCHER=1 does the same.  The
// preemption then takes the stream memory op (on ctrl_stream, or on the
// library's signal stream when ctrl_stream is NULL).
bool watcher_disabled() {
  static const bool off = getenv("NV_COMPUTE_PROFILER_PERFWORKS_DIR") != nullptr ||
                          (getenv("CTXB_NO_WATCHER") && atoi(getenv("CTXB_NO_WATCHER")) != 0);
  return off;
}

int launch_watcher(ctxb_run* r) {
  Probe* P = nullptr;
  {
    std::lock_guard<std::mutex> g(probe_mu);
    if (int rc = probe_module(r->ctx, &P)) return rc;
  }
  Driver& d = driver();
  // the watcher's "started" word: in the drain-notice page (its counter is at
  // offset 0), away from the gather words that a resume launch resets
  CUdeviceptr hw = r->hflag_dev + 32, flag = r->flag, started = r->flag + r->rep_off - FLAG_STRIDE + 128,
              stamp = r->stamps_watch, exits = r->flag + r->rep_off - FLAG_STRIDE;
  uint32_t seq = r->gate_seq, sig = r->sig, base = r->drain_base, nblk = r->grid;
  unsigned long long rep = r->rep_off;
  void* a[] = {&hw, &seq, &flag, &rep, &sig, &started, &stamp, &exits, &base, &nblk};
  CU(d.cuLaunchKernel(P->watch, 1, 1, 1, 32, 1, 1, 0, r->arm, a, nullptr));
  CU(d.cuStreamWaitValue32(r->stream, started, seq, CU_STREAM_WAIT_VALUE_GEQ));
  r->watching = true;
  return CTXB_OK;
}

// Restore-floor probe: generated per slot size, like a restore stub --
// straight-line evict-first v4 loads of every 512 B group (lane l's 16 B at
// +16 l) and v1 loads of the 1-3 trailing 128 B rows, all issued before any
// value is used, then an XOR reduction; stamps {entry, all loads back}.
std::string floor_src(uint32_t slot) {
  std::ostringstream o;
  const uint32_t ng = slot / 512, nt = (slot % 512) / 128;
  o << "typedef unsigned int u32; typedef unsigned long long u64;\n"
       "static __device__ __forceinline__ u64 gt() { u64 t; asm volatile(\"mov.u64 %0, %%globaltimer;\" : \"=l\"(t)); return t; }\n"
       "extern \"C\" __global__ void ctxb_probe_read(const unsigned char* ctx, u64* st, u32* out, u32 zero) {\n"
       "  const u32 lane = threadIdx.x & 31u, gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;\n"
       "  const u64 t0 = gt();\n"
       "  const unsigned char* p = ctx + (u64)gw * " << slot << "ull;\n";
  for (uint32_t g = 0; g < ng; g++)
    o << "  const uint4 q" << g << " = __ldcs(reinterpret_cast<const uint4*>(p + " << g * 512 << "u) + lane);\n";
  for (uint32_t t = 0; t < nt; t++)
    o << "  const u32 r" << t << " = __ldcs(reinterpret_cast<const u32*>(p + " << ng * 512 + t * 128 << "u) + lane);\n";
  o << "  u32 acc = 0u";
  for (uint32_t g = 0; g < ng; g++) o << " ^ q" << g << ".x ^ q" << g << ".y ^ q" << g << ".z ^ q" << g << ".w";
  for (uint32_t t = 0; t < nt; t++) o << " ^ r" << t;
  o << ";\n  acc = __reduce_xor_sync(0xffffffffu, acc);\n"
       "  u64 t1 = 0;\n  if ((acc & zero) == 0u) t1 = gt();\n"
       "  if (lane == 0u) { st[(u64)gw * 2] = t0; st[(u64)gw * 2 + 1] = t1; out[gw] = acc; }\n}\n";
  return o.str();
}

int floor_kernel(CUcontext c, uint32_t slot, CUfunction* fn) {
  static std::map<std::pair<CUcontext, uint32_t>, CUfunction> cache;
  auto it = cache.find({c, slot});
  if (it != cache.end()) {
    *fn = it->second;
    return CTXB_OK;
  }
  Nvrtc& n = nvrtc();
  if (!n.ok) return fail(CTXB_E_NVRTC, n.err);
  std::string src = floor_src(slot);
  void* prog = nullptr;
  if (n.CreateProgram(&prog, src.c_str(), "floor.cu", 0, nullptr, nullptr)) return fail(CTXB_E_NVRTC, "floor probe");
  const char* opts[] = {"--gpu-architecture=sm_100a"};
  if (n.CompileProgram(prog, 1, opts)) {
    n.DestroyProgram(&prog);
    return fail(CTXB_E_NVRTC, "floor probe compile");
  }
  size_t cs = 0;
  n.GetCUBINSize(prog, &cs);
  std::vector<char> cubin(cs);
  n.GetCUBIN(prog, cubin.data());
  n.DestroyProgram(&prog);
  Driver& d = driver();
  CUmodule mod = nullptr;
  CU(d.cuModuleLoadData(&mod, cubin.data()));
  CU(d.cuModuleGetFunction(fn, mod, "ctxb_probe_read"));
  cache[{c, slot}] = *fn;
  return CTXB_OK;
}

int launch(ctxb_run* r, bool resume) {
  r->sig = ++r->sig_seq;
  if (r->sig == 0) r->sig = ++r->sig_seq;   // 0 is the flags' initial value
  r->drain_base = r->drain_total;           // every block of this launch counts out once
  r->drain_total += r->grid;
  std::vector<uint64_t> blob;
  r->resumed_launch = resume;
  pack_params(r, r->prog, blob);
  void* args[] = {blob.data()};
  Driver& d = driver();
  if ((r->prog->opt.flags & CTXB_WATCHER) && !watcher_disabled()) {
    r->gate_seq = (r->gate_seq + 1) & 0x7FFFFFFFu;
    if (r->gate_seq == 0) r->gate_seq = 1;   // 0 is the host word's initial value
    if (int rc = launch_watcher(r)) return rc;
  }
  CU(d.cuEventRecord(r->ev0, r->stream));
  CU(d.cuLaunchKernel(resume ? r->mod.resume : r->mod.run, r->grid, 1, 1, (unsigned)r->prog->prog.block, 1, 1, 0,
                      r->stream, args, nullptr));
  CU(d.cuEventRecord(r->ev1, r->stream));
  if (r->prog->opt.flags & CTXB_ARMED_SIGNAL) {
    // pre-enqueue the signal behind a gate in mapped host memory: ctxb_preempt
    // only stores the gate value, no driver call on the preemption path
    r->gate_seq++;
    CU(d.cuStreamWaitValue32(r->arm, r->hflag_dev + 64, r->gate_seq, CU_STREAM_WAIT_VALUE_GEQ));
    CU(d.cuEventRecord(r->evf, r->arm));
    if (int rc = write_signal(r, r->arm)) return rc;
    r->armed = true;
  }
  r->state = RUN_RUNNING;
  r->resumed_launch = resume;
  return CTXB_OK;
}

// Read the header array after the stream drained and classify the run.
int collect(ctxb_run* r) {
  Driver& d = driver();
  r->disarm();
  if (r->hflag && (r->prog->opt.flags & CTXB_HOST_SIGNAL))   // the launch ended: lower a host word left raised
    *static_cast<volatile uint32_t*>(r->hflag) = 0u;
  r->hdr_prev.swap(r->hdr);
  r->hdr.resize((size_t)r->n_warps * 4);
  CU(d.cuMemcpyDtoHAsync(r->hdr_pin, r->cbuf, (size_t)r->n_warps * 16, r->stream));
  CU(d.cuStreamSynchronize(r->stream));
  memcpy(r->hdr.data(), r->hdr_pin, (size_t)r->n_warps * 16);
  uint32_t pre = 0, done = 0;
  for (uint32_t w = 0; w < r->n_warps; w++) {
    const uint32_t* h = &r->hdr[(size_t)w * 4];
    if (h[2] == CTXB_STATE_PREEMPTED && h[3] == r->epoch) pre++;
    else if (h[2] == CTXB_STATE_DONE) done++;
  }
  if (pre + done != r->n_warps)
    return fail(CTXB_E_CUDA, "kernel did not report every warp (" + std::to_string(pre + done) + "/" +
                                 std::to_string(r->n_warps) + "): it faulted or was not launched");
  r->state = pre ? RUN_PREEMPTED : RUN_DONE;
  return CTXB_OK;
}

// Classify a launch that ctxb_preempt left drained but not collected.
int settle(const ctxb_run* cr) {
  ctxb_run* r = const_cast<ctxb_run*>(cr);
  return r->state == RUN_DRAINED ? collect(r) : CTXB_OK;
}

template <class T>
int copy_out(const std::string& s, T* buf, size_t cap, size_t* len) {
  if (!len) return fail(CTXB_E_INVALID_ARG, "len is NULL");
  *len = s.size() + 1;
  if (!buf || cap < s.size() + 1) return fail(CTXB_E_BUFFER_TOO_SMALL, "buffer too small");
  memcpy(buf, s.c_str(), s.size() + 1);
  return CTXB_OK;
}

}  // namespace

void free_program(ctxb_program* p) {
  Driver& d = driver();
  if (d.ok) {
    for (auto& [c, m] : p->mods) d.cuModuleUnload(m.mod);
    for (auto& r : p->pool) {
      d.cuMemFree(r.flag);
      d.cuMemFree(r.stamps);
      d.cuMemFree(r.forced);
      d.cuEventDestroy(r.ev0);
      d.cuEventDestroy(r.ev1);
      d.cuEventDestroy(r.evf);
      if (r.hflag) d.cuMemFreeHost(r.hflag);
      if (r.arm) d.cuStreamDestroy(r.arm);
      if (r.hdr_pin) d.cuMemFreeHost(r.hdr_pin);
    }
  }
  delete p;
}

// IR instructions on the shortest cycle of the CFG through the basic block of
// a poll site, over every site (0 = no site lies on a loop): how often a warp
// meets a poll, the input of the poll-test cost model below.
static uint32_t shortest_poll_loop(const Program& P, const std::vector<int>& sites) {
  const size_t nb = P.bbs.size();
  auto size = [&](size_t b) { return (uint64_t)(P.bbs[b].second - P.bbs[b].first); };
  std::vector<uint8_t> seen(nb, 0);
  uint64_t best = UINT64_MAX;
  for (int c : sites) {
    if (c < 0 || (size_t)c >= P.bb_of.size()) continue;
    const size_t b0 = (size_t)P.bb_of[c];
    if (seen[b0]) continue;
    seen[b0] = 1;
    // Dijkstra from b0's successors; the weight of entering a block is its size
    std::vector<uint64_t> dist(nb, UINT64_MAX);
    std::vector<uint8_t> done(nb, 0);
    for (int s2 : P.succ[b0]) dist[s2] = std::min(dist[s2], size(s2));
    for (;;) {
      size_t u = nb;
      for (size_t v = 0; v < nb; v++)
        if (!done[v] && dist[v] != UINT64_MAX && (u == nb || dist[v] < dist[u])) u = v;
      if (u == nb || u == b0) break;
      done[u] = 1;
      for (int v : P.succ[u]) dist[v] = std::min(dist[v], dist[u] + size(v));
    }
    best = std::min(best, dist[b0]);
  }
  return best == UINT64_MAX ? 0u : (uint32_t)std::min<uint64_t>(best, UINT32_MAX);
}

// Default signal path and poll test: the watcher warp relays
// the host's store to the flag (~2 us instead of the ~7 us stream memory op)
// and the last warp's drain notice tells the host (P:74 signal, P:54-56
// drain), unless the caller chose a signal path; a synchronous flag test
// (detection within one site interval) unless the sites lie on short loops,
// where one L2 round trip per visit costs several percent and the pipelined
// test polls one of the flag replicas instead (dense polls of a large grid
// would queue on one L2 slice).
static uint32_t default_signal_flags(const Options& o, uint32_t poll_loop) {
  uint32_t f = 0;
  if (!(o.flags & (CTXB_WATCHER | CTXB_ARMED_SIGNAL | CTXB_HOST_SIGNAL))) f |= CTXB_WATCHER | CTXB_DRAIN_NOTICE;
  if (!(o.flags & (CTXB_SYNC_POLL | CTXB_FLAG_REPLICAS)) && o.flag_depth <= 1 && o.load_every <= 1)
    f |= (poll_loop && poll_loop < CTXB_DENSE_POLL_INSTRS) ? CTXB_FLAG_REPLICAS : CTXB_SYNC_POLL;
  return f;
}

extern "C" {

const char* ctxb_last_error(void) { return g_err.c_str(); }
const char* ctxb_version(void) { return "ctxb 0.1 (sm_100a, CTXB-R1)"; }

int ctxb_analyze(const char* ir_text, size_t len, const ctxb_options* opts, ctxb_program** out) {
  if (!ir_text || !out) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  *out = nullptr;
  ctxb_options o = opts ? *opts : ctxb_options{CTXB_ALL, CTXB_MODE_CTXBACK, CTXB_POLL_EVERY_INSTR, 8, 0, 1, 0, 8, 512, 0, 1};
  if (o.mode > 3 || o.poll_policy > 2 || o.flags > 65535 || ((o.flags & 2048u) && (o.flags & 4096u)) ||
      ((o.flags & CTXB_ARMED_SIGNAL) && (o.flags & CTXB_WATCHER)) || o.flag_depth > 8 || o.load_every > 1024 ||
      o.min_blocks_per_sm > 32)
    return fail(CTXB_E_INVALID_ARG, "bad options");
  std::unique_ptr<ctxb_program> p(new ctxb_program);
  p->opt = Options{o.flags, o.mode, o.poll_policy, o.poll_every ? o.poll_every : 8, o.debug,
                   o.flag_depth ? o.flag_depth : 1, o.min_blocks_per_sm,
                   o.defer_instr_bytes ? o.defer_instr_bytes : 8,
                   o.resume_level_bytes ? o.resume_level_bytes : 512, o.exact_budget,
                   o.load_every ? o.load_every : 1};
  try {
    double t0 = now_ms();
    p->prog = parse_ir(std::string(ir_text, len));
    // Gathered resume by default for kernels with atomics:
    // there the already-resumed warps' atomics fill the memory pipeline and
    // the last warps' restores queue behind them (C4a: 45-130 us tails), so
    // every resumed warp waits until all preempted warps have restored.  The
    // policy is the framework's, so the FULL / LIVE baselines get it too.
    bool atomics = false;
    for (const Instr& I : p->prog.ins) atomics = atomics || I.op == Op::AtomAdd || I.op == Op::AtomCas;
    if (atomics && !(o.debug & CTXB_DEBUG_NO_AUTO_GATHER)) p->opt.flags |= CTXB_GATHER_RESUME;
    p->an = analyze(p->prog, p->opt);
    p->poll_loop = shortest_poll_loop(p->prog, p->an.sites);
    if (!(o.debug & (CTXB_DEBUG_FORCED | CTXB_DEBUG_NO_POLLS | CTXB_DEBUG_NO_AUTO_SIGNAL)) && !p->an.sites.empty())
      p->opt.flags |= default_signal_flags(p->opt, p->poll_loop);
    double t1 = now_ms();
    p->src = generate_cuda(p->prog, p->an, p->opt, &p->cg);
    double t2 = now_ms();
    p->t_an = t1 - t0;
    p->t_cg = t2 - t1;
  } catch (const ParseError& e) {
    return fail(CTXB_E_PARSE, e.what());
  } catch (const std::exception& e) {
    return fail(CTXB_E_ANALYSIS, std::string("analysis: ") + e.what());
  }
  if (!(o.debug & CTXB_DEBUG_NO_COMPILE)) {
    double t0 = now_ms();
    int rc = compile(p.get());
    if (rc) return rc;
    p->t_cc = now_ms() - t0;
  }
  *out = p.release();
  return CTXB_OK;
}

int ctxb_program_destroy(ctxb_program* p) {
  if (!p) return fail(CTXB_E_INVALID_ARG, "NULL program");
  {
    std::lock_guard<std::mutex> g(p->mu);
    if (p->live_runs > 0) {   // freed by the last run's destructor
      p->destroy_pending = true;
      return CTXB_OK;
    }
  }
  free_program(p);
  return CTXB_OK;
}


int ctxb_program_info(const ctxb_program* p, ctxb_program_info_t* o) {
  if (!p || !o) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  o->n_instrs = (uint32_t)p->prog.ins.size();
  o->nv = (uint32_t)p->prog.nv;
  o->ns = (uint32_t)p->prog.ns;
  o->block = (uint32_t)p->prog.block;
  o->n_buffers = (uint32_t)p->prog.buf_names.size();
  o->n_uniforms = (uint32_t)p->prog.uniforms.size();
  o->n_sites = (uint32_t)p->an.sites.size();
  o->n_backups = (uint32_t)p->an.backups.size();
  o->max_payload_bytes_per_warp = p->cg.max_payload;
  o->full_ir_bytes_per_warp = p->an.full_ir_bytes;
  o->num_regs = p->num_regs;
  o->compiled = p->cubin.empty() ? 0 : 1;
  o->num_regs_resume = p->regs_resume;
  o->resume_maxnreg = p->cg.resume_maxnreg;
  o->n_save_stubs = p->cg.n_save_stubs;
  o->cubin_bytes = (uint32_t)p->cubin.size();
  o->exact_windows = p->an.exact_windows;
  o->exact_truncated = p->an.exact_truncated;
  o->exact_improved = p->an.exact_improved;
  o->exact_fallback = p->an.exact_fallback;
  o->analyze_ms = p->t_an;
  o->codegen_ms = p->t_cg;
  o->compile_ms = p->t_cc;
  o->spill_stores = p->spill_st;
  o->spill_loads = p->spill_ld;
  o->spill_stores_resume = p->spill_st_res;
  o->spill_loads_resume = p->spill_ld_res;
  o->gather_resume = (p->opt.flags & CTXB_GATHER_RESUME) ? 1u : 0u;
  o->n_fp_shared = p->cg.n_fp_shared;
  o->flags = p->opt.flags;
  o->poll_loop_instrs = p->poll_loop;
  return CTXB_OK;
}

int ctxb_program_cubin(const ctxb_program* p, void* buf, size_t cap, size_t* len) {
  if (!p || !len) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (p->cubin.empty()) return fail(CTXB_E_STATE, "program was analysed with CTXB_DEBUG_NO_COMPILE");
  *len = p->cubin.size();
  if (!buf || cap < p->cubin.size()) return fail(CTXB_E_BUFFER_TOO_SMALL, "buffer too small");
  memcpy(buf, p->cubin.data(), p->cubin.size());
  return CTXB_OK;
}

int ctxb_num_sites(const ctxb_program* p, uint32_t* n) {
  if (!p || !n) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  *n = (uint32_t)p->an.sites.size();
  return CTXB_OK;
}

int ctxb_site_info(const ctxb_program* p, uint32_t site, ctxb_site_info_t* o) {
  if (!p || !o) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (site >= p->an.sites.size()) return fail(CTXB_E_INVALID_ARG, "site out of range");
  const Plan& pl = p->an.plans[site];
  o->c = (uint32_t)pl.c;
  o->p = (uint32_t)pl.p;
  o->n_vec = pl.n_vec;
  o->n_scalar = pl.n_sca;
  o->n_revert_pre = pl.n_rev_pre;
  o->n_revert_res = pl.n_rev_res;
  o->n_reexec = pl.n_reexec;
  o->payload_bytes_per_warp = pl.payload_bytes;
  o->live_bytes_per_warp = p->an.live[site].payload_bytes;
  o->defer_site = (uint32_t)p->an.defer[site];
  o->reexec_load_bytes_per_warp = 0;
  for (const Event& e : pl.schedule)
    if (e.is_x && p->prog.ins[e.j].op == Op::Ldg)
      o->reexec_load_bytes_per_warp += p->prog.is_vec(p->prog.ins[e.j].defreg) ? 128u : 4u;
  return CTXB_OK;
}

int ctxb_backups(const ctxb_program* p, uint32_t* idx, uint32_t cap, uint32_t* n) {
  if (!p || !n) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  *n = (uint32_t)p->an.backups.size();
  for (uint32_t i = 0; i < *n && i < cap && idx; i++) idx[i] = (uint32_t)p->an.backups[i];
  return CTXB_OK;
}

int ctxb_site_plan_text(const ctxb_program* p, uint32_t site, int live, char* buf, size_t cap, size_t* len) {
  if (!p) return fail(CTXB_E_INVALID_ARG, "NULL program");
  if (site >= p->an.sites.size()) return fail(CTXB_E_INVALID_ARG, "site out of range");
  return copy_out(plan_text(p->prog, live ? p->an.live[site] : p->an.plans[site]), buf, cap, len);
}

int ctxb_generated_source(const ctxb_program* p, char* buf, size_t cap, size_t* len) {
  if (!p) return fail(CTXB_E_INVALID_ARG, "NULL program");
  return copy_out(p->src, buf, cap, len);
}

int ctxb_occupancy(ctxb_program* p, uint32_t* bps, uint32_t* nsm) {
  if (!p || !bps || !nsm) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  CUcontext c;
  int rc = ensure_ctx(&c);
  if (rc) return rc;
  Mod m;
  rc = ensure_module(p, c, &m);
  if (rc) return rc;
  Driver& d = driver();
  int a = 0, b = 0, n = 0;
  CU(d.cuOccupancyMaxActiveBlocksPerMultiprocessor(&a, m.run, p->prog.block, 0));
  CU(d.cuOccupancyMaxActiveBlocksPerMultiprocessor(&b, m.resume, p->prog.block, 0));
  CUdevice dev;
  CU(d.cuCtxGetDevice(&dev));
  CU(d.cuDeviceGetAttribute(&n, CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, dev));
  *bps = (uint32_t)std::min(a, b);
  *nsm = (uint32_t)n;
  return CTXB_OK;
}

int ctxb_persistent_grid(ctxb_program* p, uint32_t* grid) {
  if (!p || !grid) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  uint32_t bps = 0, nsm = 0;
  if (int rc = ctxb_occupancy(p, &bps, &nsm)) return rc;
  *grid = bps * nsm;
  if (!(p->opt.flags & CTXB_WATCHER) || bps == 0) return CTXB_OK;
  // the watcher warp (32 threads, its registers, no shared memory) must fit
  // on one SM next to bps blocks, else that SM hosts one block fewer
  CUcontext c;
  if (int rc = ensure_ctx(&c)) return rc;
  Probe* P = nullptr;
  {
    std::lock_guard<std::mutex> g(probe_mu);
    if (int rc = probe_module(c, &P)) return rc;
  }
  Mod m;
  if (int rc = ensure_module(p, c, &m)) return rc;
  Driver& d = driver();
  int rw = 0, rv = 0, rr = 0, sv = 0, sr = 0, smem_sm = 0, maxw = 0;
  CUdevice dev;
  CU(d.cuCtxGetDevice(&dev));
  CU(d.cuFuncGetAttribute(&rw, CU_FUNC_ATTRIBUTE_NUM_REGS, P->watch));
  CU(d.cuFuncGetAttribute(&rv, CU_FUNC_ATTRIBUTE_NUM_REGS, m.run));
  CU(d.cuFuncGetAttribute(&rr, CU_FUNC_ATTRIBUTE_NUM_REGS, m.resume));
  CU(d.cuFuncGetAttribute(&sv, CU_FUNC_ATTRIBUTE_SHARED_SIZE_BYTES, m.run));
  CU(d.cuFuncGetAttribute(&sr, CU_FUNC_ATTRIBUTE_SHARED_SIZE_BYTES, m.resume));
  CU(d.cuDeviceGetAttribute(&smem_sm, CU_DEVICE_ATTRIBUTE_MAX_SHARED_MEMORY_PER_MULTIPROCESSOR, dev));
  CU(d.cuDeviceGetAttribute(&maxw, CU_DEVICE_ATTRIBUTE_MAX_THREADS_PER_MULTIPROCESSOR, dev));
  auto warp_regs = [](int r) { return ((r * 32 + 255) / 256) * 256; };
  const uint32_t wpb = p->prog.block / 32;
  const uint64_t regs = (uint64_t)bps * wpb * (uint64_t)warp_regs(std::max(rv, rr)) + warp_regs(rw);
  const uint64_t warps = (uint64_t)bps * wpb + 1;
  const uint64_t smem = (uint64_t)bps * (uint64_t)(std::max(sv, sr) + 1024);
  if (regs > 65536 || warps > (uint64_t)maxw / 32 || bps + 1 > 32 || smem > (uint64_t)smem_sm) *grid -= 1;
  return CTXB_OK;
}

int ctxb_context_capacity(const ctxb_program* p, uint32_t grid, uint64_t* bytes) {
  if (!p || !bytes || grid == 0) return fail(CTXB_E_INVALID_ARG, "bad argument");
  if (p->opt.mode == CTXB_MODE_FULL_HW && p->num_regs == 0)
    return fail(CTXB_E_STATE, "FULL_HW capacity needs the compiled register count");
  uint64_t nw = (uint64_t)grid * (p->prog.block / 32);
  uint64_t off = ((nw * 16 + 255) / 256) * 256;
  *bytes = off + nw * p->stride();
  return CTXB_OK;
}

int ctxb_launch(ctxb_program* p, uint32_t grid, void* const* buffers, const uint32_t* uniforms, void* ctx_buf,
                uint64_t ctx_bytes, void* stream, const uint32_t* forced_targets, ctxb_run** out) {
  if (!p || !out || grid == 0) return fail(CTXB_E_INVALID_ARG, "bad argument");
  *out = nullptr;
  if (!p->prog.buf_names.empty() && !buffers) return fail(CTXB_E_INVALID_ARG, "buffers is NULL");
  if (!p->prog.uniforms.empty() && !uniforms) return fail(CTXB_E_INVALID_ARG, "uniforms is NULL");
  if (!ctx_buf) return fail(CTXB_E_INVALID_ARG, "ctx_buf is NULL");
  CUcontext c;
  int rc = ensure_ctx(&c);
  if (rc) return rc;
  std::unique_ptr<ctxb_run> r(new ctxb_run);
  r->prog = p;
  {
    std::lock_guard<std::mutex> g(p->mu);
    p->live_runs++;
  }
  r->ctx = c;
  rc = ensure_module(p, c, &r->mod);
  if (rc) return rc;
  uint64_t need = 0;
  rc = ctxb_context_capacity(p, grid, &need);
  if (rc) return rc;
  if (ctx_bytes < need)
    return fail(CTXB_E_BUFFER_TOO_SMALL, "context buffer has " + std::to_string(ctx_bytes) + " bytes, needs " +
                                             std::to_string(need));
  Driver& d = driver();
  r->grid = grid;
  r->n_warps = grid * (p->prog.block / 32);
  for (size_t i = 0; i < p->prog.buf_names.size(); i++) r->bufs.push_back((uint64_t)(uintptr_t)buffers[i]);
  for (size_t i = 0; i < p->prog.uniforms.size(); i++) r->uni.push_back(uniforms[i]);
  r->cbuf = (CUdeviceptr)(uintptr_t)ctx_buf;
  r->cbytes = ctx_bytes;
  r->pay_off = (((uint64_t)r->n_warps * 16 + 255) / 256) * 256;
  r->stride = p->stride();
  r->stream = (CUstream)stream;
  {
    std::lock_guard<std::mutex> g(p->mu);
    for (size_t i = 0; i < p->pool.size(); i++)
      if (p->pool[i].n_warps == r->n_warps) {
        r->flag = p->pool[i].flag;
        r->stamps = p->pool[i].stamps;
        r->forced = p->pool[i].forced;
        r->ev0 = p->pool[i].ev0;
        r->ev1 = p->pool[i].ev1;
        r->evf = p->pool[i].evf;
        r->hflag = p->pool[i].hflag;
        r->hflag_dev = p->pool[i].hflag_dev;
        r->arm = p->pool[i].arm;
        r->gate_seq = p->pool[i].gate_seq;
        r->hdr_pin = p->pool[i].hdr_pin;
        r->rep_off = p->pool[i].rep_off;
        r->sig_seq = p->pool[i].sig_seq;
        r->drain_total = p->pool[i].drain_total;
        p->pool.erase(p->pool.begin() + (long)i);
        break;
      }
  }
  if (!r->flag) {
    CUdeviceptr f = 0, s = 0, t = 0;
    // flag (+0), gather arrivals (+128), a gather release word per block (+256);
    // then FLAG_REPLICAS replicas, one per 4 KiB page (rep_off)
    // (+ one page for the drain-notice exit counter, just below the replicas)
    r->rep_off = ((256 + (uint64_t)grid * 4 + FLAG_STRIDE - 1) / FLAG_STRIDE) * FLAG_STRIDE + FLAG_STRIDE;
    CU(d.cuMemAlloc(&f, r->rep_off + (size_t)FLAG_REPLICAS * FLAG_STRIDE));
    CU(d.cuMemAlloc(&s, (size_t)r->n_warps * 32 + 64));   // + the watcher's stamp
    CU(d.cuMemsetD8Async(s + (CUdeviceptr)r->n_warps * 32, 0, 64, nullptr));
    CU(d.cuMemAlloc(&t, (size_t)r->n_warps * 4));
    r->flag = f;
    r->stamps = s;
    r->forced = t;
    CU(d.cuEventCreate(&r->ev0, CU_EVENT_DEFAULT));
    CU(d.cuEventCreate(&r->ev1, CU_EVENT_DEFAULT));
    CU(d.cuEventCreate(&r->evf, CU_EVENT_DEFAULT));
    CU(d.cuMemHostAlloc(&r->hdr_pin, (size_t)r->n_warps * 16, 0));
    std::vector<uint8_t> z(r->rep_off + (size_t)FLAG_REPLICAS * FLAG_STRIDE, 0);
    CU(d.cuMemcpyHtoD(r->flag, z.data(), z.size()));   // the flags are 0 whenever a run does not hold them raised
  }
  if (!r->hflag) {   // [0] host signal word, [16] armed gate, [24] drain notice
    void* h = nullptr;
    CU(d.cuMemHostAlloc(&h, 128, CU_MEMHOSTALLOC_DEVICEMAP | CU_MEMHOSTALLOC_PORTABLE));
    memset(h, 0, 128);
    r->hflag = h;
    CU(d.cuMemHostGetDevicePointer(&r->hflag_dev, h, 0));
  }
  r->stamps_watch = r->stamps + (CUdeviceptr)r->n_warps * 32;
  if ((p->opt.flags & (CTXB_ARMED_SIGNAL | CTXB_WATCHER)) && !r->arm) {
    int lo = 0, hi = 0;
    CU(d.cuCtxGetStreamPriorityRange(&lo, &hi));
    CU(d.cuStreamCreateWithPriority(&r->arm, CU_STREAM_NON_BLOCKING, hi));
  }
  // No header memset: every warp of launch 0 writes its header (DONE or
  // PREEMPTED with epoch 1) before the launch completes.
  rc = upload_forced(r.get(), forced_targets);
  if (rc) return rc;
  r->epoch = 1;
  rc = launch(r.get(), false);
  if (rc) return rc;
  *out = r.release();
  return CTXB_OK;
}

// The signal must not be ordered behind the victim kernel, or it would arrive
// only once the kernel has finished (and "preempt" would silently wait for
// natural completion).  Unless the signal is pre-enqueued on the library's own
// non-blocking stream (CTXB_ARMED_SIGNAL), reject: ctrl == the run's stream;
// ctrl == the legacy default stream (NULL / CU_STREAM_LEGACY), which waits for
// every blocking stream; and a blocking ctrl stream when the run itself is on
// the legacy default stream.
static int check_ctrl(const ctxb_run* r, void* ctrl) {
  if (r->armed) return CTXB_OK;
  // CTXB_WATCHER with ctrl == NULL: the watcher alone (or, where no watcher
  // runs, the memop on the library's own non-blocking signal stream)
  if ((r->prog->opt.flags & CTXB_WATCHER) && ctrl == nullptr) return CTXB_OK;
  CUstream cs = (CUstream)ctrl, rs = r->stream;
  if (cs == rs) return fail(CTXB_E_INVALID_ARG, "ctrl_stream must differ from the run's stream");
  if (cs == nullptr || cs == CU_STREAM_LEGACY)
    return fail(CTXB_E_INVALID_ARG, "ctrl_stream is the legacy default stream, which is ordered behind the "
                                    "victim kernel: pass a non-blocking stream");
  if (rs == nullptr || rs == CU_STREAM_LEGACY) {
    unsigned fl = 0;
    CU(driver().cuStreamGetFlags(cs, &fl));
    if (!(fl & CU_STREAM_NON_BLOCKING))
      return fail(CTXB_E_INVALID_ARG, "the run is on the legacy default stream and ctrl_stream is a blocking "
                                      "stream, so the signal would wait for the victim: use non-blocking streams");
  }
  return CTXB_OK;
}

int ctxb_preempt(ctxb_run* r, void* ctrl, ctxb_preempt_stats* st) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  if (r->state != RUN_RUNNING) return fail(CTXB_E_STATE, "run is not running");
  if (int rc = check_ctrl(r, ctrl)) return rc;
  Driver& d = driver();
  volatile uint32_t* hf =
      (r->prog->opt.flags & CTXB_HOST_SIGNAL) ? static_cast<volatile uint32_t*>(r->hflag) : nullptr;
  double t0 = now_ms();
  if (hf) {
    // CTXB_HOST_SIGNAL: relay warps see this store over PCIe and raise the
    // device flag; the stream memory op below stays as the fallback (every
    // relay warp may have finished already)
    *hf = 1u;
    std::atomic_thread_fence(std::memory_order_seq_cst);
  }
  // CTXB_WATCHER: the co-resident watcher warp sees this store over PCIe and
  // raises the device flags; the stream memory op stays as the fallback
  const bool watch = r->watching;
  if (watch) {
    *(static_cast<volatile uint32_t*>(r->hflag) + 8) = r->gate_seq;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    r->watching = false;
  }
  // test knob: CTXB_HOST_SIGNAL_ONLY=1 drops the fallback, so the relay (or
  // the watcher) is the only path
  const char* ho = (hf || watch) ? getenv("CTXB_HOST_SIGNAL_ONLY") : nullptr;
  const bool host_only = ho && atoi(ho) != 0;
  CUstream cs = (CUstream)ctrl;
  const bool no_fallback = (hf || watch) && (host_only || ctrl == nullptr);
  if (!watch && !cs && (r->prog->opt.flags & CTXB_WATCHER)) cs = r->arm;   // no watcher ran (profiler)
  if (r->armed) {
    // CTXB_ARMED_SIGNAL: release the signal enqueued on the library's stream at launch
    *(static_cast<volatile uint32_t*>(r->hflag) + 16) = r->gate_seq;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    r->armed = false;
    cs = r->arm;
  } else {
    if (!no_fallback) {
      CU(d.cuEventRecord(r->evf, cs));
      if (int rc = write_signal(r, cs)) return rc;
    }
  }
  // env CTXB_PREEMPT_TIMEOUT_US > 0: give up waiting for the drain after that
  // long (a kernel without reachable poll sites); the signal stays raised and
  // the run stays running (ctxb_wait / ctxb_query later see how it ended)
  const char* te = getenv("CTXB_PREEMPT_TIMEOUT_US");
  const double tmo_us = te ? atof(te) : 0.0;
  // Drained = the last warp's drain notice (host word [24] == this launch's
  // signal value, written over PCIe as it exits) or the launch's end event,
  // whichever the host sees first; the event is queried every ~256 spins.
  volatile uint32_t* drain = static_cast<volatile uint32_t*>(r->hflag) + 24;
  const bool notice = r->prog->opt.flags & CTXB_DRAIN_NOTICE;
  if (!notice && tmo_us <= 0.0) CU(d.cuStreamSynchronize(r->stream));
  for (uint32_t it = 0; notice || tmo_us > 0.0; it++) {
    if (notice && *drain == r->sig) break;
    if ((it & 255u) == 255u) {
      CUresult q = d.cuEventQuery(r->ev1);
      if (q == CUDA_SUCCESS) break;
      if (q != CUDA_ERROR_NOT_READY) return fail(CTXB_E_CUDA, "cuEventQuery: " + cu_err(q));
      if (tmo_us > 0.0 && (now_ms() - t0) * 1e3 > tmo_us)
        return fail(CTXB_E_TIMEOUT, "the run did not drain within CTXB_PREEMPT_TIMEOUT_US (signal left raised)");
    }
  }
  double t1 = now_ms();
  if (hf) *hf = 0u;   // the victim has drained: no warp of this run reads it until the next launch
  if (!st) {
    // return at once: the headers are read when first needed (settle)
    r->state = RUN_DRAINED;
    return CTXB_OK;
  }
  if (cs) CU(d.cuStreamSynchronize(cs));   // the signal stream (none: watcher without fallback)
  int rc = collect(r);
  if (rc) return rc;
  {
    memset(st, 0, sizeof *st);
    st->host_us = (t1 - t0) * 1e3;
    std::vector<uint64_t> stamps((size_t)r->n_warps * 4);
    CU(d.cuMemcpyDtoH(stamps.data(), r->stamps, stamps.size() * 8));
    uint64_t tmin = UINT64_MAX, tmax = 0;
    std::vector<uint8_t> blk(r->grid, 0);
    uint32_t nwb = r->prog->prog.block / 32;
    for (uint32_t w = 0; w < r->n_warps; w++) {
      const uint32_t* h = &r->hdr[(size_t)w * 4];
      if (h[2] == CTXB_STATE_PREEMPTED && h[3] == r->epoch) {
        st->warps_preempted++;
        st->payload_bytes += h[1];
        st->header_bytes += 16;
        blk[w / nwb] = 1;
        tmin = std::min(tmin, stamps[(size_t)w * 4 + 0]);
        tmax = std::max(tmax, stamps[(size_t)w * 4 + 1]);
      } else if (h[2] == CTXB_STATE_DONE) {
        st->warps_done++;
      }
    }
    for (auto b : blk) st->blocks_preempted += b;
    st->latency_us = st->warps_preempted ? (double)(tmax - tmin) * 1e-3 : 0.0;
    float ms = 0;
    if (!(hf || watch)) CU(d.cuEventElapsedTime(&ms, r->evf, r->ev1));
    // with CTXB_HOST_SIGNAL / CTXB_WATCHER the signal is the host store, which the event does not bound
    st->signal_to_drained_us = (hf || watch) ? 0.0 : (double)ms * 1e3;
  }
  return CTXB_OK;
}

int ctxb_preempt_async(ctxb_run* r, void* ctrl) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  if (r->state != RUN_RUNNING) return fail(CTXB_E_STATE, "run is not running");
  if (int rc = check_ctrl(r, ctrl)) return rc;
  Driver& d = driver();
  if (r->prog->opt.flags & CTXB_HOST_SIGNAL) {   // lowered when the launch is collected
    *static_cast<volatile uint32_t*>(r->hflag) = 1u;
    std::atomic_thread_fence(std::memory_order_seq_cst);
  }
  const bool watched = r->watching;
  if (r->watching) {   // CTXB_WATCHER: the watcher relays the host store (the memop stays as the fallback)
    *(static_cast<volatile uint32_t*>(r->hflag) + 8) = r->gate_seq;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    r->watching = false;
  }
  if (r->armed) {
    *(static_cast<volatile uint32_t*>(r->hflag) + 16) = r->gate_seq;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    r->armed = false;
  } else if (!(watched && ctrl == nullptr)) {
    CUstream cs = (ctrl == nullptr && (r->prog->opt.flags & CTXB_WATCHER)) ? r->arm : (CUstream)ctrl;
    CU(d.cuEventRecord(r->evf, cs));
    if (int rc = write_signal(r, cs)) return rc;
  }
  // the run stays RUNNING: ctxb_wait / ctxb_query see it drain (PREEMPTED or DONE)
  return CTXB_OK;
}

int ctxb_resume(ctxb_run* r, void* stream, const uint32_t* forced_targets) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  if (int rc = settle(r)) return rc;
  if (r->state != RUN_PREEMPTED) return fail(CTXB_E_STATE, "run is not preempted");
  r->stream = (CUstream)stream;
  int rc = upload_forced(r, forced_targets);
  if (rc) return rc;
  r->rb_target = 0;
  if (r->prog->opt.flags & CTXB_GATHER_RESUME) {
    // wait only for warps that can all be resident at once (persistent grid)
    // blocks that can all be resident at once (a static property of the
    // program on this context: computed once, off the later resumes' path)
    uint64_t resident = 0;
    {
      std::lock_guard<std::mutex> g(r->prog->mu);
      auto it = r->prog->gather_resident.find(r->ctx);
      if (it != r->prog->gather_resident.end()) resident = it->second;
    }
    if (!resident) {
      Driver& d = driver();
      int b = 0, n = 0;
      CUdevice dev;
      CU(d.cuOccupancyMaxActiveBlocksPerMultiprocessor(&b, r->mod.resume, r->prog->prog.block, 0));
      CU(d.cuCtxGetDevice(&dev));
      CU(d.cuDeviceGetAttribute(&n, CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, dev));
      resident = (uint64_t)b * (uint64_t)n;
      if ((r->prog->opt.flags & CTXB_WATCHER) && !watcher_disabled()) {
        // the watcher warp takes a slot: a block that cannot be resident beside
        // it would keep the gathered blocks waiting
        uint32_t g = 0;
        if (int rc = ctxb_persistent_grid(r->prog, &g)) return rc;
        resident = std::min<uint64_t>(resident, g);
      }
      std::lock_guard<std::mutex> g(r->prog->mu);
      r->prog->gather_resident[r->ctx] = resident;
    }
    if ((uint64_t)r->grid <= resident) {
      // target = blocks with >= 1 preempted warp (one global arrival per block)
      uint32_t nwb = r->prog->prog.block / 32, blocks = 0;
      for (uint32_t b = 0; b < r->grid; b++) {
        bool any = false;
        for (uint32_t w = b * nwb; w < (b + 1) * nwb; w++)
          any = any || (r->hdr[(size_t)w * 4 + 2] == CTXB_STATE_PREEMPTED && r->hdr[(size_t)w * 4 + 3] == r->epoch);
        blocks += any;
      }
      r->rb_target = blocks;
      CU(driver().cuMemsetD32Async(r->flag + 128, 0, 32 + r->grid, r->stream));   // arrivals + release words
    }
  }
  r->epoch++;
  return launch(r, true);
}

int ctxb_wait(ctxb_run* r, int* finished) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  if (int rc = settle(r)) return rc;
  if (r->state == RUN_RUNNING) {
    r->release_watcher();
    CU(driver().cuStreamSynchronize(r->stream));
    int rc = collect(r);
    if (rc) return rc;
  }
  if (finished) *finished = r->state == RUN_DONE ? 1 : 0;
  return CTXB_OK;
}

int ctxb_query(ctxb_run* r, int* running) {
  if (!r || !running) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (int rc = settle(r)) return rc;
  if (r->state != RUN_RUNNING) {
    *running = 0;
    return CTXB_OK;
  }
  CUresult q = driver().cuEventQuery(r->ev1);
  if (q == CUDA_ERROR_NOT_READY) {
    *running = 1;
    return CTXB_OK;
  }
  if (q != CUDA_SUCCESS) return fail(CTXB_E_CUDA, "cuEventQuery: " + cu_err(q));
  int rc = collect(r);
  if (rc) return rc;
  *running = 0;
  return CTXB_OK;
}

// ---- flag propagation probe (measured separately) -------------


int ctxb_restore_floor(void* stream, uint32_t bytes_per_warp, uint32_t grid_blocks, uint32_t block,
                       uint32_t trials, double* median_us) {
  if (!median_us || trials == 0 || grid_blocks == 0 || block == 0 || block % 32 || block > 1024 ||
      bytes_per_warp == 0 || bytes_per_warp % 128 || bytes_per_warp > (1u << 20))
    return fail(CTXB_E_INVALID_ARG, "bad argument");
  CUcontext c;
  int rc = ensure_ctx(&c);
  if (rc) return rc;
  std::lock_guard<std::mutex> g(probe_mu);
  CUfunction read = nullptr;
  if ((rc = floor_kernel(c, bytes_per_warp, &read))) return rc;
  Driver& d = driver();
  const uint64_t nw = (uint64_t)grid_blocks * (block / 32);
  const size_t scratch_bytes = 256u << 20;   // > the 126 MB L2: every trial reads from HBM
  CUdeviceptr ctx = 0, st = 0, out = 0, scr = 0;
  CU(d.cuMemAlloc(&ctx, nw * bytes_per_warp));
  CU(d.cuMemAlloc(&st, nw * 16));
  CU(d.cuMemAlloc(&out, nw * 4));
  CU(d.cuMemAlloc(&scr, scratch_bytes));
  CUstream s = (CUstream)stream;
  std::vector<double> v;
  std::vector<uint64_t> h(nw * 2);
  int err = CTXB_OK;
  CU(d.cuMemsetD32Async(ctx, 0x5A5A5A5Au, nw * bytes_per_warp / 4, s));
  for (uint32_t t = 0; t <= trials && !err; t++) {
    uint32_t zero = 0;
    void* a[] = {&ctx, &st, &out, &zero};
    if (d.cuMemsetD32Async(scr, t, scratch_bytes / 4, s) != CUDA_SUCCESS ||
        d.cuLaunchKernel(read, grid_blocks, 1, 1, block, 1, 1, 0, s, a, nullptr) != CUDA_SUCCESS ||
        d.cuStreamSynchronize(s) != CUDA_SUCCESS || d.cuMemcpyDtoH(h.data(), st, nw * 16) != CUDA_SUCCESS) {
      err = fail(CTXB_E_CUDA, "restore floor probe failed");
      break;
    }
    uint64_t a0 = UINT64_MAX, b0 = 0;
    for (uint64_t w = 0; w < nw; w++) {
      a0 = std::min(a0, h[w * 2]);
      b0 = std::max(b0, h[w * 2 + 1]);
    }
    if (t) v.push_back((double)(b0 - a0) * 1e-3);   // the first trial is a warm-up
  }
  d.cuMemFree(ctx);
  d.cuMemFree(st);
  d.cuMemFree(out);
  d.cuMemFree(scr);
  if (err) return err;
  std::sort(v.begin(), v.end());
  *median_us = v[v.size() / 2];
  return CTXB_OK;
}

int ctxb_flag_propagation(void* ctrl, uint32_t trials, double* median_us, double* max_us) {
  if (!median_us || trials == 0) return fail(CTXB_E_INVALID_ARG, "bad argument");
  CUcontext c;
  int rc = ensure_ctx(&c);
  if (rc) return rc;
  std::lock_guard<std::mutex> g(probe_mu);
  Probe* PP = nullptr;
  if ((rc = probe_module(c, &PP))) return rc;
  Probe& P = *PP;
  Driver& d = driver();
  CUdeviceptr flag = 0, out = 0;
  CU(d.cuMemAlloc(&flag, 256));
  CU(d.cuMemAlloc(&out, 64));
  {
    // load both kernels now (CUDA lazy loading would otherwise load the stamp
    // kernel while the spinner runs, which waits for the spinner: deadlock)
    uint32_t one = 1;
    CU(d.cuMemcpyHtoD(flag, &one, 4));
    void* a1[] = {&flag, &out};
    CU(d.cuLaunchKernel(P.spin, 1, 1, 1, 32, 1, 1, 0, nullptr, a1, nullptr));
    void* a2[] = {&out};
    CU(d.cuLaunchKernel(P.stamp, 1, 1, 1, 32, 1, 1, 0, nullptr, a2, nullptr));
    CU(d.cuStreamSynchronize(nullptr));
  }
  std::vector<double> v;
  // The spinner runs on a private non-blocking stream.  Kernels on different
  // streams are not guaranteed to be co-scheduled, so no stamp kernel is put
  // in front of the flag write; instead an event on `ctrl` is recorded right
  // before the write and one on the spinner's stream right after the
  // spinner: elapsed = write issued -> spinner saw the flag and exited
  // (an upper bound; includes the kernel's exit).
  CUstream spin_s = nullptr;
  CU(d.cuStreamCreate(&spin_s, CU_STREAM_NON_BLOCKING));
  CUevent e0, e1;
  CU(d.cuEventCreate(&e0, CU_EVENT_DEFAULT));
  CU(d.cuEventCreate(&e1, CU_EVENT_DEFAULT));
  for (uint32_t t = 0; t < trials; t++) {
    uint32_t zero = 0;
    CU(d.cuMemcpyHtoD(flag, &zero, 4));
    void* a1[] = {&flag, &out};
    CU(d.cuLaunchKernel(P.spin, 1, 1, 1, 32, 1, 1, 0, spin_s, a1, nullptr));
    CU(d.cuEventRecord(e1, spin_s));
    double t0 = now_ms();
    while (now_ms() < t0 + 0.2) {
    }
    CU(d.cuEventRecord(e0, (CUstream)ctrl));
    CU(d.cuStreamWriteValue32((CUstream)ctrl, flag, 1u, 0));
    CU(d.cuStreamSynchronize((CUstream)ctrl));
    CU(d.cuStreamSynchronize(spin_s));
    float ms = 0;
    CU(d.cuEventElapsedTime(&ms, e0, e1));
    v.push_back((double)ms * 1e3);
  }
  d.cuEventDestroy(e0);
  d.cuEventDestroy(e1);
  d.cuStreamDestroy(spin_s);
  d.cuMemFree(flag);
  d.cuMemFree(out);
  std::sort(v.begin(), v.end());
  *median_us = v[v.size() / 2];
  if (max_us) *max_us = v.back();
  return CTXB_OK;
}

int ctxb_launch_ms(const ctxb_run* r, float* ms) {
  if (!r || !ms) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (int rc = settle(r)) return rc;
  if (r->state == RUN_RUNNING) return fail(CTXB_E_STATE, "launch still running: call ctxb_wait/ctxb_preempt first");
  Driver& d = driver();
  CU(d.cuEventSynchronize(r->ev1));
  CU(d.cuEventElapsedTime(ms, r->ev0, r->ev1));
  return CTXB_OK;
}

int ctxb_resume_stats_get(const ctxb_run* r, ctxb_resume_stats* o) {
  if (!r || !o) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (int rc = settle(r)) return rc;
  memset(o, 0, sizeof *o);
  if (!r->resumed_launch || r->state == RUN_RUNNING || r->hdr_prev.empty()) return CTXB_OK;
  std::vector<uint64_t> stamps((size_t)r->n_warps * 4);
  CU(driver().cuMemcpyDtoH(stamps.data(), r->stamps, stamps.size() * 8));
  uint64_t tmin = UINT64_MAX, tmax = 0;
  for (uint32_t w = 0; w < r->n_warps; w++) {
    const uint32_t* h = &r->hdr_prev[(size_t)w * 4];
    if (h[2] == CTXB_STATE_PREEMPTED && h[3] + 1 == r->epoch) {
      o->warps_resumed++;
      tmin = std::min(tmin, stamps[(size_t)w * 4 + 2]);
      tmax = std::max(tmax, stamps[(size_t)w * 4 + 3]);
    }
  }
  o->resume_us = o->warps_resumed ? (double)(tmax - tmin) * 1e-3 : 0.0;
  return CTXB_OK;
}

int ctxb_context_bytes(const ctxb_run* r, uint64_t* payload, uint64_t* header, uint32_t* n_tb) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  if (int rc = settle(r)) return rc;
  uint64_t pb = 0, hb = 0;
  uint32_t nwb = r->prog->prog.block / 32;
  std::vector<uint8_t> blk(r->grid, 0);
  for (uint32_t w = 0; w < r->n_warps && !r->hdr.empty(); w++) {
    const uint32_t* h = &r->hdr[(size_t)w * 4];
    if (h[2] == CTXB_STATE_PREEMPTED && h[3] == r->epoch) {
      pb += h[1];
      hb += 16;
      blk[w / nwb] = 1;
    }
  }
  uint32_t nt = 0;
  for (auto b : blk) nt += b;
  if (payload) *payload = pb;
  if (header) *header = hb;
  if (n_tb) *n_tb = nt;
  return CTXB_OK;
}

int ctxb_read_headers(const ctxb_run* r, uint32_t* out, uint64_t n) {
  if (!r || !out) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (int rc = settle(r)) return rc;
  if (n < (uint64_t)r->n_warps * 4) return fail(CTXB_E_BUFFER_TOO_SMALL, "need 4 words per warp");
  if (r->hdr.empty()) return fail(CTXB_E_STATE, "no completed launch yet");
  memcpy(out, r->hdr.data(), (size_t)r->n_warps * 16);
  return CTXB_OK;
}

int ctxb_read_stamps(const ctxb_run* r, uint64_t* out, uint64_t n) {
  if (!r || !out) return fail(CTXB_E_INVALID_ARG, "NULL argument");
  if (int rc = settle(r)) return rc;
  if (n < (uint64_t)r->n_warps * 4) return fail(CTXB_E_BUFFER_TOO_SMALL, "need 4 words per warp");
  // one more word: the CTXB_WATCHER stamp (when the last watcher raised the flag)
  const size_t words = (size_t)r->n_warps * 4 + (n > (uint64_t)r->n_warps * 4 ? 1 : 0);
  CU(driver().cuMemcpyDtoH(out, r->stamps, words * 8));
  return CTXB_OK;
}

int ctxb_run_destroy(ctxb_run* r) {
  if (!r) return fail(CTXB_E_INVALID_ARG, "NULL run");
  delete r;
  return CTXB_OK;
}

}  // extern "C"
