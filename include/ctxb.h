/*
 * ctxb.h -- C ABI of the B200-native CTXBack context save / restore path.
 *
 * CTXBack (Ji & Wang, IPDPS 2021; `P:n` = line n of reference PAPER.md) lets a
 * preempted warp save the register context of a *preceding* instruction (its
 * flashback-point) instead of the current one, and on resume reload that
 * context, revert and re-execute the in-between instructions.
 *
 * This library implements, for kernels written in the small register IR of
 * DESIGN.md ("IR v1"):
 *   - the compile-time pass: liveness, flashback-point search with
 *     the relaxed condition, instruction reverting and on-chip scalar backup,
 *     per-site plan selection, and generation of one dedicated preemption
 *     routine and one dedicated resume routine per poll site, as sm_100a CUDA
 *     compiled with NVRTC                                 -> ctxb_analyze
 *   - the runtime: launching the generated kernel, raising the
 *     preemption signal, draining the warps into a caller-owned context
 *     buffer, and resuming them                          -> ctxb_launch /
 *                                                           ctxb_preempt /
 *                                                           ctxb_resume
 *
 * Conventions
 *   - Every function returns an int status: CTXB_OK (0) or a negative
 *     CTXB_E_* code.  No C++ exception crosses the ABI.  ctxb_last_error()
 *     returns a thread-local message describing the last failure.
 *   - Handles (ctxb_program, ctxb_run) are created and destroyed by the
 *     library.  Device buffers and the context buffer are owned by the
 *     caller (e.g. torch tensors, passed as raw device pointers); they must
 *     outlive every run that uses them.
 *   - Streams are borrowed: `stream` arguments are CUstream / cudaStream_t
 *     handles of the current device's primary context passed as void*
 *     (NULL = legacy default stream).  No torch type appears here.
 *   - There is no CPU fallback: ctxb_launch and friends fail with
 *     CTXB_E_CUDA when no CUDA device / driver is present.  ctxb_analyze needs
 *     only NVRTC (it compiles without a GPU) unless CTXB_DEBUG_NO_COMPILE.
 */
#ifndef CTXB_H
#define CTXB_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------ */
#define CTXB_OK                  0
#define CTXB_E_INVALID_ARG      -1   /* NULL handle / out pointer, bad index, bad size   */
#define CTXB_E_PARSE            -2   /* IR text does not follow DESIGN.md "IR v1"        */
#define CTXB_E_ANALYSIS         -3   /* internal analysis failure (a bug)                */
#define CTXB_E_NVRTC            -4   /* NVRTC missing or generated CUDA failed to build  */
#define CTXB_E_CUDA             -5   /* driver missing or a CUDA driver call failed      */
#define CTXB_E_STATE            -6   /* preempt on a finished run, resume on a run that
                                        is not preempted, ...                            */
#define CTXB_E_BUFFER_TOO_SMALL -7   /* context buffer / output buffer too small         */
#define CTXB_E_TIMEOUT          -8   /* ctxb_preempt: no drain within env
                                        CTXB_PREEMPT_TIMEOUT_US; the run stays running
                                        with the signal raised                          */

/* ---- options (P:34-36 three techniques; P:337 compared schemes) ---------- */
#define CTXB_RELAXED  1u  /* relaxed flashback-point condition, Alg. 1 */
#define CTXB_REVERT   2u  /* instruction reverting, Alg. 2            */
#define CTXB_OSRB     4u  /* on-chip scalar register backup           */
#define CTXB_ALL      7u
#define CTXB_DEFER    8u  /* CS-Defer (ref [4]): a preemption arriving at a
                             site may continue to a later site of the same basic
                             block whose estimated latency is lower; combined
                             with CTXBack plans = CTXBack+CS-Defer,
                             with CTXB_MODE_LIVE = CS-Defer                       */
#define CTXB_PRUNE   16u  /* demand-driven restore (NEXT N4): restore only what the
                             registers live at the site need, instead of every
                             live-out result of the window (R-2, literal); every
                             flashback-point becomes feasible                     */
#define CTXB_RANK_RESUME 32u /* combined ranking (NEXT N4): per site pick the
                             flashback-point minimising the estimated preempt +
                             resume cost E = 2*payload + re-executed load bytes +
                             resume_level_bytes*(dependent memory round trips - 1)
                             + defer_instr_bytes*(reverts + re-executions), ties
                             by the R-10 key; the paper ranks by preemption
                             latency only and notes re-execution can dominate
                             resuming                          */
#define CTXB_EXACT   64u  /* exact plan search (NEXT N4, R-19): per
                             window, the minimum-bytes set of values saved at
                             preempt whose resume closure (re-execution and
                             reverting as an order-free fixpoint)
                             restores every required value, by branch and bound
                             seeded with the greedy CTXB-R1 plan; a window whose
                             search exceeds exact_budget nodes (or 48 candidate
                             values) keeps its greedy plan (counted in
                             ctxb_program_info_t.exact_truncated)               */

#define CTXB_GATHER_RESUME 128u /* runtime (default for kernels with atomics, see
                             CTXB_DEBUG_NO_AUTO_GATHER): in a resume launch of a persistent grid
                             (every block resident), a warp that has restored its
                             context waits until every preempted warp of the
                             launch has restored (or the flag rises again, or
                             20 us pass; env CTXB_GATHER_TIMEOUT_NS) before
                             continuing, so early warps' work does not queue the
                             late warps' restores in the memory system; off:
                             each warp continues at once                        */

#define CTXB_SYNC_POLL   256u /* codegen: a poll site tests the flag value it loads
                             itself (one L2 round trip per poll) instead of the
                             value loaded flag_depth sites earlier: detection
                             within one site interval instead of flag_depth + 1,
                             for loops whose iterations are long (C4a)         */
#define CTXB_HOST_SIGNAL 512u /* (A/B study option, superseded by the default
                             CTXB_WATCHER path of DESIGN.md 8q.)
                             runtime + codegen: ctxb_preempt also raises a word
                             in mapped pinned host memory.  Each warp reads it
                             (system-scope load over PCIe, tested one site
                             later) once every ceil(n_warps / R) of its polls,
                             staggered by warp id (R = env CTXB_HOST_RELAYS,
                             default 1: ~R reads per poll interval device-wide)
                             and forwards a raised word to the device flag
                             that every warp polls; the stream memory op is
                             still issued as the fallback (env
                             CTXB_HOST_SIGNAL_ONLY=1 drops it: tests).  Cuts the signal's
                             ~7.6 us stream-memop path.  Flag
                             mode only (ignored by CTXB_DEBUG_FORCED).
                             stats.signal_to_drained_us is 0 in this mode (the
                             host store is not stream-ordered): use host_us   */
#define CTXB_ARMED_SIGNAL 1024u /* (A/B option, superseded by the default CTXB_WATCHER
                             path of DESIGN.md 8q: -12 µs host latency on C2.)
                             runtime: every launch (and resume) pre-enqueues
                             its preemption signal on a library-owned
                             greatest-priority stream: cuStreamWaitValue32 on a
                             gate word in mapped pinned host memory, then the
                             signal event and cuStreamWriteValue32(flag).
                             ctxb_preempt then only stores the gate value (no
                             driver call on the preemption path; ctrl_stream
                             is not used); a launch that completes unpreempted
                             is disarmed when it is collected (ctxb_wait /
                             ctxb_query / destroy).  Kernels are unchanged.
                             signal_to_drained_us = signal event (after the
                             gate opened) -> victim drained    */
#define CTXB_OSRB_SMEM  2048u /* codegen: OSRB backups live in a
                             per-warp shared-memory slot (the paper's LDS
                             tier: 4 B per backup per warp) instead of a
                             register (4 B per backup per thread); lane 0
                             stores the warp-uniform value, the preemption
                             routine reads it after __syncwarp().  Plans and
                             bytes unchanged                                  */
#define CTXB_OSRB_LANES 4096u /* (A/B option: slower than the default register slot,
                             DESIGN.md 8k.)
                             codegen: OSRB backup j lives in lane j % 32 of one
                             register per 32 backups (the paper's VGPR-lane
                             tier), read back with a warp shuffle in the
                             (converged) preemption routine.  Exclusive with
                             CTXB_OSRB_SMEM (_INVALID_ARG).  Plans unchanged  */
#define CTXB_FLAG_REPLICAS 8192u /* codegen: one warp in max(1, n_warps / 32)
                             polls the master flag word, the others one of 64
                             replicas (one per 4 KiB page, so dense polls of a
                             large grid spread over L2 slices instead of
                             queueing on one); a master poller that sees the
                             signal forwards it to every replica; replica
                             pollers read the master at every 64th load (so
                             finished master pollers cannot hide a signal).
                             Detection takes up to one more poll interval
                             (none with CTXB_WATCHER, which raises the master
                             and every replica itself).  For kernels with
                             frequent polls (C3: 0.90 -> 0.24 ms)            */
#define CTXB_DRAIN_NOTICE 16384u /* codegen + runtime: the launch's last warp to
                             exit writes its signal value to a word in mapped
                             pinned host memory (one shared-memory count per
                             block, one global atomic per block), and
                             ctxb_preempt returns when it sees that word
                             instead of the kernel's completion event: host
                             latency -5 µs on C2, but the kernel's completion
                             (the sysmem write is flushed at kernel end) comes
                             ~2 µs later.  The per-block exit
                             count alone is also kept for CTXB_WATCHER       */

#define CTXB_WATCHER 32768u /* runtime: every launch (and resume) first starts a
                             one-warp watcher kernel on a library-owned
                             greatest-priority stream; the launch waits (stream
                             memory op) until it runs, so it is co-resident with
                             the victim (ctxb_persistent_grid leaves room for
                             it).  ctxb_preempt stores the launch's sequence
                             number to a word in mapped pinned host memory; the
                             watcher polls that word with system-scope loads and
                             raises the device flag (+ replicas), bypassing the
                             ~7 us stream memory op, which stays as the fallback
                             on ctrl_stream (ctrl_stream == NULL, or env
                             CTXB_HOST_SIGNAL_ONLY=1, drops it).  A launch that ends unpreempted
                             releases its watcher when collected.
                             signal_to_drained_us is 0 (the host store is not
                             stream-ordered): use host_us.  Exclusive with
                             CTXB_ARMED_SIGNAL (_INVALID_ARG).  No watcher is
                             started under Nsight Compute or with env
                             CTXB_NO_WATCHER=1 (the memop is then the signal,
                             on the library's stream if ctrl_stream is NULL)  */

#define CTXB_MODE_CTXBACK 0u /* per site: least-context flashback-point */
#define CTXB_MODE_LIVE    1u /* save LIVE_IN(site) (ref [4])              */
#define CTXB_MODE_FULL    2u /* save every declared IR register (FULL_IR)        */
#define CTXB_MODE_FULL_HW 3u /* FULL_IR padded to the compiled kernel's register
                                count per thread: the analogue of the BASELINE
                                routine that swaps all occupied registers */

#define CTXB_POLL_EVERY_INSTR 0u /* a poll site before every IR instruction   */
#define CTXB_POLL_EVERY_N     1u /* before BB-local index i, i % N == 0, i > 0,
                                    and before every backward branch          */
#define CTXB_POLL_EXPLICIT    2u /* before the IR's `poll` markers             */

#define CTXB_DEBUG_FORCED     1u /* poll sites compare the warp's poll-visit count
                                    with a per-warp target instead of reading the
                                    preemption flag (deterministic tests)      */
#define CTXB_DEBUG_POISON     2u /* the resume kernel fills every IR register with
                                    a poison pattern before restoring          */
#define CTXB_DEBUG_NO_POLLS   4u /* compile poll sites out (overhead baseline;
                                    the kernel cannot be preempted)            */
#define CTXB_DEBUG_NO_COMPILE 8u /* analysis + code generation only            */
#define CTXB_DEBUG_NO_SHARE  16u /* one preemption routine per site (no P:317
                                    sharing at all)                            */
#define CTXB_DEBUG_NO_AUTO_GATHER 128u /* do not turn CTXB_GATHER_RESUME on by
                                    default for kernels with atomics (A/B)     */
#define CTXB_DEBUG_NO_FP_SHARE 256u /* keep only the exact sharing of byte-identical
                                    preemption routines: no per-flashback-point
                                    routine with entry offsets (A/B)    */
#define CTXB_DEBUG_NO_SPEC_RESTORE 512u /* no speculative restore loads: the
                                    resume kernel issues the payload loads only
                                    after the header's dispatch (A/B; by default
                                    up to 16 registers of payload common to every
                                    site's layout are loaded with the header)   */
#define CTXB_DEBUG_NO_AUTO_SIGNAL 1024u /* keep exactly the caller's signal-path
                                    and poll-test bits.  By default a program
                                    with flag-mode poll sites (not _FORCED, not
                                    _NO_POLLS) gets:
                                    * CTXB_WATCHER | CTXB_DRAIN_NOTICE unless the
                                      caller chose a signal path (CTXB_WATCHER,
                                      CTXB_ARMED_SIGNAL or CTXB_HOST_SIGNAL);
                                    * the poll test from a cost model, unless the
                                      caller chose one (CTXB_SYNC_POLL,
                                      CTXB_FLAG_REPLICAS, flag_depth > 1 or
                                      load_every > 1): a site on a loop of fewer
                                      than CTXB_DENSE_POLL_INSTRS IR instructions
                                      -> CTXB_FLAG_REPLICAS with the pipelined
                                      test (a synchronous test would add an L2
                                      round trip to every short iteration);
                                      otherwise CTXB_SYNC_POLL.
                                    ctxb_program_info_t.flags reports the result */
#define CTXB_DENSE_POLL_INSTRS 32u
#define CTXB_DEBUG_FENCE_STAMPS 32u /* __threadfence before the t_saved stamp, so
                                    it marks the payload as visible (slower
                                    drain; by default the kernel boundary orders
                                    the context for the resume launch)          */

typedef struct {
  uint32_t flags;       /* CTXB_RELAXED | CTXB_REVERT | CTXB_OSRB                */
  uint32_t mode;        /* CTXB_MODE_*                                           */
  uint32_t poll_policy; /* CTXB_POLL_*                                           */
  uint32_t poll_every;  /* N for CTXB_POLL_EVERY_N                               */
  uint32_t debug;       /* CTXB_DEBUG_* bits                                     */
  uint32_t flag_depth;  /* flag-load pipeline depth D >= 1 (0 = 1): a poll site
                           tests the flag value loaded D sites earlier, hiding the
                           L2 round trip behind D site intervals (dense sites ->
                           larger D)                                              */
  uint32_t min_blocks_per_sm; /* 0 = compiler's choice; else both generated kernels
                           get __launch_bounds__(block, n): ptxas caps registers
                           so n blocks fit per SM (persistent-grid occupancy)      */
  uint32_t defer_instr_bytes; /* CTXB_DEFER latency estimate: one deferred instruction
                           costs this many context bytes (0 = 8); the stalls of the
                           deferred instructions are ignored, as in P:380          */
  uint32_t resume_level_bytes; /* CTXB_RANK_RESUME: one dependent memory round trip on
                           the resume path costs this many context bytes per warp
                           (0 = 512 ~ an HBM round trip x one warp's share of HBM
                           bandwidth when every warp of the chip restores)        */
  uint32_t exact_budget; /* CTXB_EXACT: branch-and-bound nodes per window (0 = 2^20) */
  uint32_t load_every;  /* flag mode: a warp loads the flag at every K-th poll visit
                           (0 = 1) and tests the last loaded value at the others:
                           K times fewer flag loads for kernels with very dense
                           polls, detection up to K - 1 visits later          */
} ctxb_options;

typedef struct ctxb_program ctxb_program; /* analysed IR kernel + module; library-owned */
typedef struct ctxb_run ctxb_run;         /* one launch and its preempt/resume history   */

/* Per poll-site plan summary (one dedicated routine pair per site). */
typedef struct {
  uint32_t c;               /* site = before IR instruction c (R-1)           */
  uint32_t p;               /* chosen flashback-point instruction (p <= c)          */
  uint32_t n_vec;           /* saved vector values (128 B per warp each, R-8)       */
  uint32_t n_scalar;        /* saved scalar values (4 B per warp each)              */
  uint32_t n_revert_pre;    /* reverting instructions run at preempt (Alg. 2)       */
  uint32_t n_revert_res;    /* reverting instructions run at resume                 */
  uint32_t n_reexec;        /* re-executed instructions at resume (Alg. 1)          */
  uint32_t payload_bytes_per_warp; /* 128*n_vec + 4*n_scalar                        */
  uint32_t live_bytes_per_warp;    /* the LIVE plan of the same site (fallback)     */
  uint32_t defer_site;             /* CTXB_DEFER: site a preemption arriving here is
                                      carried to (== this site: no deferral)          */
  uint32_t reexec_load_bytes_per_warp; /* bytes the resume's re-executed loads read per
                                      warp (128 B vector / 4 B scalar each): memory
                                      traffic of the replay beside the payload      */
} ctxb_site_info_t;

typedef struct {
  uint32_t n_instrs, nv, ns, block, n_buffers, n_uniforms, n_sites, n_backups;
  uint32_t max_payload_bytes_per_warp; /* over every plan incl. LIVE fallbacks       */
  uint32_t full_ir_bytes_per_warp;     /* 128*nv + 4*ns                              */
  uint32_t num_regs;                   /* ptxas registers/thread (0 if not compiled) */
  uint32_t compiled;                   /* 1 if a cubin was produced                  */
  uint32_t num_regs_resume;            /* ptxas registers/thread of the resume kernel */
  uint32_t resume_maxnreg;             /* min blocks/SM requested for the resume kernel
                                          (__launch_bounds__) so it keeps the normal
                                          kernel's occupancy (0 = none needed)       */
  uint32_t n_save_stubs;               /* distinct preemption-routine bodies after
                                          sharing                            */
  uint32_t cubin_bytes;                /* size of the compiled sm_100a cubin         */
  uint32_t exact_windows;              /* CTXB_EXACT: (site, flashback-point) windows
                                          searched                                    */
  uint32_t exact_truncated;            /*   of which the search was cut off (budget or
                                          > 48 candidates): greedy plan kept          */
  uint32_t exact_improved;             /*   of which the exact plan saves fewer bytes
                                          than the greedy CTXB-R1 plan                */
  uint32_t exact_fallback;             /*   greedy kept although the search completed
                                          (never expected; a consistency check)       */
  double analyze_ms, codegen_ms, compile_ms;
  uint32_t spill_stores, spill_loads;  /* ptxas -v spill bytes of the normal kernel (0 if the
                                          log was not produced, e.g. under ncu)     */
  uint32_t spill_stores_resume, spill_loads_resume;   /* same for ctxb_resume      */
  uint32_t gather_resume;              /* 1 if resume launches gather (CTXB_GATHER_RESUME
                                          given, or chosen by default because the
                                          kernel has atomics)                        */
  uint32_t n_fp_shared;                /* sites whose preemption routine is their
                                          flashback-point's shared routine, entered at
                                          an offset past the later sites' reverts */
  uint32_t flags;                      /* the option bits in effect: the caller's plus
                                          those ctxb_analyze chose by default
                                          (CTXB_GATHER_RESUME, and the signal path and
                                          poll test of CTXB_DEBUG_NO_AUTO_SIGNAL)     */
  uint32_t poll_loop_instrs;           /* IR instructions on the shortest loop through
                                          a poll site (0 = no site lies on a loop):
                                          the poll-test cost model's input           */
} ctxb_program_info_t;

typedef struct {
  double latency_us;         /* device: max t_saved - min t_flag_seen over preempted
                                warps (%globaltimer): the preemption routines'
                                span (t_saved = stores issued; with
                                CTXB_DEBUG_FENCE_STAMPS: stores visible)          */
  double host_us;            /* host: flag write issued -> victim stream drained   */
  double signal_to_drained_us; /* CUDA events: event on ctrl right before the flag
                                write -> the library's event after the victim
                                kernel (every warp saved or done, kernel exited);
                                negative if the kernel had finished already     */
  uint32_t warps_preempted, warps_done, blocks_preempted;
  uint64_t payload_bytes;    /* sum of saved payload over preempted warps          */
  uint64_t header_bytes;     /* 16 B per preempted warp                             */
} ctxb_preempt_stats;

typedef struct {
  double resume_us;          /* device: max t_site_reached - min t_resume_entry    */
  uint32_t warps_resumed;
} ctxb_resume_stats;

const char* ctxb_last_error(void);
const char* ctxb_version(void);

/* Parse + analyse + generate + compile.  `ir_text` need not be
 * NUL-terminated (`len` bytes are read).  opts == NULL means
 * {CTXB_ALL, CTXB_MODE_CTXBACK, CTXB_POLL_EVERY_INSTR, 8, 0, 1, 0, 8, 512, 0, 1}.
 * Errors: _INVALID_ARG, _PARSE, _ANALYSIS, _NVRTC. */
int ctxb_analyze(const char* ir_text, size_t len, const ctxb_options* opts, ctxb_program** out);
/* Release the program.  Runs that still reference it keep it alive: the last
 * run's ctxb_run_destroy frees it (any destruction order is safe). */
int ctxb_program_destroy(ctxb_program* prog);
int ctxb_program_info(const ctxb_program* prog, ctxb_program_info_t* out);
int ctxb_num_sites(const ctxb_program* prog, uint32_t* n);
int ctxb_site_info(const ctxb_program* prog, uint32_t site, ctxb_site_info_t* out);
/* OSRB-selected scalar defs (instruction indices), up to `cap`; *n = total. */
int ctxb_backups(const ctxb_program* prog, uint32_t* idx, uint32_t cap, uint32_t* n);
/* Canonical text of a site's plan, NUL-terminated;
 * *len = required size incl. NUL; _BUFFER_TOO_SMALL if cap < *len. */
int ctxb_site_plan_text(const ctxb_program* prog, uint32_t site, int live, char* buf, size_t cap,
                        size_t* len);
/* The generated CUDA C++ source (same buffer convention). */
int ctxb_generated_source(const ctxb_program* prog, char* buf, size_t cap, size_t* len);
/* The compiled sm_100a cubin (ELF) of the program's two kernels (the normal and
 * the resume kernel) -- the output of the compile-time pass with
 * its dedicated routines: *len = its size; copied to caller-owned `buf` if
 * cap >= *len, else _BUFFER_TOO_SMALL.  _STATE if compiled with
 * CTXB_DEBUG_NO_COMPILE; _INVALID_ARG on NULL prog / len.  Lets a caller
 * inspect the generated code with its own tools (cuobjdump -sass,
 * --dump-resource-usage) independently of this library. */
int ctxb_program_cubin(const ctxb_program* prog, void* buf, size_t cap, size_t* len);

/* Resident blocks per SM of the generated kernels (min over the normal and the
 * resume kernel, driver occupancy calculator) and the device's SM count: a
 * persistent grid is blocks_per_sm * num_sms ("persistent thread").
 * Needs a GPU (_CUDA otherwise). */
int ctxb_occupancy(ctxb_program* prog, uint32_t* blocks_per_sm, uint32_t* num_sms);

/* The largest grid whose blocks are all resident at once ("persistent
 * thread"): blocks_per_sm * num_sms, one block fewer when the program uses
 * CTXB_WATCHER and the watcher warp does not fit next to blocks_per_sm
 * blocks on an SM (registers of the larger of the two kernels, warps, blocks,
 * shared memory).  A persistent kernel launched with more blocks still runs
 * correctly, but its extra block waits for a free slot (a doubled tail).
 * Needs a GPU (_CUDA otherwise); _INVALID_ARG on NULL arguments. */
int ctxb_persistent_grid(ctxb_program* prog, uint32_t* grid);

/* Bytes of device memory a context buffer for `grid_blocks` blocks needs:
 * 16 B header per warp + per-warp payload slots. */
int ctxb_context_capacity(const ctxb_program* prog, uint32_t grid_blocks, uint64_t* bytes);

/* Launch the generated kernel ("if no preemption occurs, CTXBack incurs
 * no extra work except OSRB").  buffers[i] = device pointer of the i-th
 * `.buffer` in IR order (u32 elements); uniforms[i] = value of the i-th
 * `.uniform`.  ctx_buf: caller-owned device memory of >= capacity bytes.
 * forced_targets (CTXB_DEBUG_FORCED programs only, else NULL): host array of
 * grid_blocks*block/32 u32, the 0-based poll visit at which each warp is
 * preempted (0xFFFFFFFF = never).  The launch is asynchronous on `stream`. */
int ctxb_launch(ctxb_program* prog, uint32_t grid_blocks, void* const* buffers,
                const uint32_t* uniforms, void* ctx_buf, uint64_t ctx_buf_bytes, void* stream,
                const uint32_t* forced_targets, ctxb_run** out);

/* Raise the preemption signal and wait until every warp of the run has
 * either saved its context and exited or finished.  Flags are never
 * reset: the next launch waits for a different value.  Fills `stats` if
 * non-NULL.  stats == NULL returns as soon as the launch drained; the headers
 * are read by the next call that needs the run's state (ctxb_wait / query /
 * resume / read_*), so the GPU is free for other work one host round trip
 * earlier.  _STATE if the run is not running. */
/* Signal paths: by default (CTXB_WATCHER) a host store that the
 * launch's watcher warp relays to the flag words; ctrl_stream may be NULL (the
 * watcher alone) or a stream that also issues the stream-memop write as a
 * fallback.  Otherwise the launch's unique signal value is written to the
 * master flag word by `ctrl_stream` (which must not be the run's stream, nor
 * the legacy stream, nor a blocking stream while the run is on the legacy
 * stream: _INVALID_ARG), or with CTXB_ARMED_SIGNAL by the library's own
 * stream; polling warps forward it to the flag replicas they poll.  With
 * CTXB_DRAIN_NOTICE (default with the watcher) the wait ends on the last
 * warp's store to host memory. */
int ctxb_preempt(ctxb_run* run, void* ctrl_stream, ctxb_preempt_stats* stats);

/* Raise the preemption signal and return at once (no drain wait): the host
 * can launch the latency-sensitive work right away and the block scheduler
 * starts it as the preempted blocks exit.  The run stays running until
 * ctxb_wait / ctxb_query observe the drain (then PREEMPTED or DONE, as after
 * ctxb_preempt).  _STATE if the run is not running. */
int ctxb_preempt_async(ctxb_run* run, void* ctrl_stream);

/* Relaunch the same grid as a resume kernel: each preempted warp reloads its
 * context, reverts / re-executes to its site and continues; finished warps
 * exit at once.  forced_targets as in ctxb_launch.  Asynchronous.
 * _STATE unless the run is preempted. */
int ctxb_resume(ctxb_run* run, void* stream, const uint32_t* forced_targets);

/* Wait for the run's current launch; *finished = 1 if every warp is done,
 * 0 if some warps were preempted (forced mode or a racing ctxb_preempt). */
int ctxb_wait(ctxb_run* run, int* finished);

/* Non-blocking: *running = 1 while the run's current launch is executing;
 * once it has completed, the headers are collected (as ctxb_wait does) and
 * *running = 0.  Lets a host scheduler poll a batch job between arrivals. */
int ctxb_query(ctxb_run* run, int* running);

/* Propagation time of the preemption signal: a one-warp spinner polls a flag
 * (ld.relaxed.gpu, like the poll sites); an event is recorded on `ctrl` right
 * before the flag is written by cuStreamWriteValue32 on `ctrl` (exactly as
 * ctxb_preempt does) and another after the spinner on its own stream; result
 * = elapsed time between the two (an upper bound: includes the spinner's
 * exit).  Median / max over `trials` (added to the drain
 * latency as a separately measured constant).  Needs an idle GPU. */
int ctxb_flag_propagation(void* ctrl_stream, uint32_t trials, double* median_us, double* max_us);

/* Cold-read floor of a restore (measurement probe): a kernel of
 * grid_blocks x block threads in which every warp reads its own
 * bytes_per_warp-byte slot with the context layout's evict-first 128-bit
 * loads and XOR-reduces it, L2 evicted before each trial (256 MiB written on
 * `stream`); result = median over `trials` of (max over warps of "all loads
 * returned" - min over warps of entry), %globaltimer, the definition of the
 * resume time.  It is what a resume of that many bytes per warp on that grid
 * costs with no dispatch, replay or register pressure.  bytes_per_warp must
 * be a multiple of 128.  Allocates (and frees) its buffers; needs an idle GPU. */
int ctxb_restore_floor(void* stream, uint32_t bytes_per_warp, uint32_t grid_blocks, uint32_t block,
                       uint32_t trials, double* median_us);

/* Duration of the run's last kernel launch (normal or resume), from CUDA
 * events the library records immediately before and after cuLaunchKernel on
 * the launching stream.  Valid after ctxb_wait / ctxb_preempt returned. */
int ctxb_launch_ms(const ctxb_run* run, float* ms);

/* Device timings of the last resume launch (valid after ctxb_wait/preempt). */
int ctxb_resume_stats_get(const ctxb_run* run, ctxb_resume_stats* out);

/* Sum over warps of the last preemption: payload bytes, header bytes and the
 * number of thread blocks with >= 1 preempted warp (P:343 context size). */
int ctxb_context_bytes(const ctxb_run* run, uint64_t* payload, uint64_t* header,
                       uint32_t* n_tb_preempted);

/* Copy the per-warp headers {site | live<<31, payload_bytes, state, epoch}
 * (4 u32 per warp) of the last completed launch into host memory. */
int ctxb_read_headers(const ctxb_run* run, uint32_t* host_out, uint64_t n_words);
/* Copy the per-warp %globaltimer stamps {t_flag_seen, t_saved, t_resume_entry,
 * t_site_reached} (4 u64 per warp).  With n_words > 4 x warps one more word
 * follows: the %globaltimer at which the run's CTXB_WATCHER warp last raised
 * the flag (0 if it never did). */
int ctxb_read_stamps(const ctxb_run* run, uint64_t* host_out, uint64_t n_words);

/* Release the run handle; its device resources return to the program's pool.
 * A launch that is still running is waited for first (not preempted).  The
 * caller's buffers and context buffer are not freed (caller-owned). */
int ctxb_run_destroy(ctxb_run* run);

/* Header `state` values. */
#define CTXB_STATE_NONE      0u
#define CTXB_STATE_PREEMPTED 1u
#define CTXB_STATE_DONE      2u

#ifdef __cplusplus
}
#endif
#endif /* CTXB_H */
