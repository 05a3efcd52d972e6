// runtime.cu — the C ABI (include/rtlsim.h): context lifecycle, device
// memory, the per-chunk schedule and the pipelined stimulus upload / output
// drain.
//
// PAPER.md mapping:
//   * CUDA Graph execution (§3.2.2): the per-cycle partition
//     schedule is either one fused chunk kernel that walks every partition's
//     steps for Tc cycles per launch (default: no per-cycle launch at all), or,
//     with RTLSIM_F_GRAPH, Tc x P per-(cycle, partition) kernel nodes captured
//     once into a CUDA graph and replayed.
//   * Pipeline scheduling (§3.2.3): stimulus chunks are uploaded
//     and transposed (N2) on one side stream while the previous chunk is
//     simulated and the one before is transposed back (N3) and drained on
//     another; double-buffered, chained by events.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <vector>

#include "../../include/rtlsim.h"
#include <dlfcn.h>

#include "jit.h"
#include "kernels.h"
#include "program.h"

using namespace rtlsim;

namespace {
thread_local std::string g_load_error;

enum SrcKind { SRC_NONE = 0, SRC_HOST, SRC_DEVICE, SRC_PRODUCER };

struct Dest {
  uint32_t *out_host = nullptr, *out_dev = nullptr;
  uint64_t *dig_host = nullptr, *dig_dev = nullptr;
  rtlsim_consumer cons = nullptr;
  void *user = nullptr;
  uint64_t cycles = 0;   // total cycles of this run (output pitch)
};

bool is_pinned(const void *p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost;
}
}  // namespace

struct rtlsim_ctx {
  Program prog;
  rtlsim_options opt{};
  bool host_only = false, failed = false;
  std::string err;
  int device = 0;
  cudaStream_t st = nullptr, st_h2d = nullptr, st_d2h = nullptr;
  bool own_stream = false;
  uint32_t smem_bytes = 0;
  uint64_t launches = 0;
  uint64_t device_bytes = 0;
  std::vector<void *> dev_allocs;     // freed at rtlsim_free
  std::vector<void *> bind_allocs;    // freed at re-bind
  std::vector<void *> host_allocs;    // pinned, freed at re-bind
  // static device data
  uint4 *d_desc = nullptr, *d_bitdesc = nullptr;
  uint32_t *d_bitptr = nullptr, *d_stepwait = nullptr;
  WideRec *d_wide = nullptr;
  uint32_t *d_step = nullptr, *d_consts = nullptr, *d_mask = nullptr, *d_reginit = nullptr;
  RegWord *d_regmap = nullptr;
  // binding
  SrcKind src = SRC_NONE;
  const uint32_t *stim = nullptr;
  bool stim_pinned = false;
  rtlsim_producer prod = nullptr;
  void *prod_user = nullptr;
  uint64_t N = 0, T = 0, cycle = 0, cycle0_run = 0;
  uint64_t static_bytes = 0;
  uint32_t N_pad = 0, Tc = 64;
  Arena state[2]{}, xnet{};
  Arena d_in[2]{};                    // class-formatted input rows [Tc][rows][N]
  InStride in_stride{};
  RegWord *d_inmap = nullptr;
  uint32_t *d_cov = nullptr;          // RTLSIM_F_COVERAGE: [RW] toggle bitmap (N5)
  uint32_t *d_mem = nullptr;          // memories: [MR][N_pad] u32 (per-stimulus entries)
  uint32_t *d_port = nullptr;         // write-port words of the current cycle [PW][N_pad]
  MemPortDev *d_ports = nullptr;      // port descriptors (static)
  uint32_t *d_meminit = nullptr;      // [MR] initial row values (static)
  uint32_t *d_out[2]{}, *d_raw[2]{}, *d_outu[2]{};
  unsigned long long *d_dig[2]{}, *d_digu[2]{};
  uint32_t *h_in[2]{}, *h_out[2]{};
  unsigned long long *h_dig[2]{};
  cudaEvent_t ev_in_ready[2]{}, ev_comp_done[2]{}, ev_drain_done[2]{}, ev_h2d_copied[2]{}, ev_start = nullptr;
  bool ev_used[2] = {false, false};
  std::map<uint64_t, cudaGraphExec_t> graphs;   // graph mode: key (buf, parity, nc)
  // RTLSIM_F_TIMING: event pairs around evaluator launches, folded lazily
  struct Timed {
    cudaEvent_t a, b;
    uint64_t stim_cycles;
  };
  std::vector<Timed> timed_pending;
  std::vector<cudaEvent_t> event_pool;
  double eval_ms = 0;
  uint64_t eval_launches = 0, eval_stim_cycles = 0;
  JitKernels jit;        // RTLSIM_F_JIT (no digest code)
  JitKernels jit_dig;    // RTLSIM_F_JIT check-mode variant, built on the first digest run
  std::string jit_rt_path;
  uint32_t jit_smem = 0, jit_smem_cap = 0;
  // concurrent per-cycle graph: fork / join streams and per-partition events
  std::vector<cudaStream_t> dag_streams;
  std::vector<cudaEvent_t> dag_events;
  cudaEvent_t dag_fork = nullptr;
};

#define CK(call)                                                                       \
  do {                                                                                 \
    cudaError_t e_ = (call);                                                           \
    if (e_ != cudaSuccess) return cuda_fail(ctx, e_, #call, __LINE__);                 \
  } while (0)

// JIT kernels specialised for the bound N_pad (state-row offsets as
// immediates, jit.cpp gaddr) unless RTLSIM_JIT_GENERIC is set (A/B)
static bool jit_specialise() { return getenv("RTLSIM_JIT_GENERIC") == nullptr; }

static int cuda_fail(rtlsim_ctx *ctx, cudaError_t e, const char *what, int line) {
  ctx->failed = true;
  ctx->err = std::string("CUDA error ") + cudaGetErrorString(e) + " at runtime.cu:" + std::to_string(line) +
             " (" + what + ")";
  return RTLSIM_E_CUDA;
}

static int arg_fail(rtlsim_ctx *ctx, int code, const std::string &msg) {
  ctx->err = msg;
  return code;
}

static cudaError_t dalloc(rtlsim_ctx *ctx, void **p, size_t bytes, bool bind_scope) {
  *p = nullptr;
  if (bytes == 0) return cudaSuccess;
  cudaError_t e = cudaMalloc(p, bytes);
  if (e != cudaSuccess) return e;
  ctx->device_bytes += bytes;
  (bind_scope ? ctx->bind_allocs : ctx->dev_allocs).push_back(*p);
  return cudaSuccess;
}

static void free_binding(rtlsim_ctx *ctx) {
  for (void *p : ctx->bind_allocs) cudaFree(p);
  ctx->bind_allocs.clear();
  for (void *p : ctx->host_allocs) cudaFreeHost(p);
  ctx->host_allocs.clear();
  for (auto &kv : ctx->graphs) cudaGraphExecDestroy(kv.second);
  ctx->graphs.clear();
  for (int b = 0; b < 2; b++) {
    ctx->d_in[b] = Arena{};
    ctx->d_out[b] = ctx->d_raw[b] = ctx->d_outu[b] = nullptr;
    ctx->d_dig[b] = ctx->d_digu[b] = nullptr;
    ctx->h_in[b] = ctx->h_out[b] = nullptr;
    ctx->h_dig[b] = nullptr;
    ctx->ev_used[b] = false;
  }
  ctx->d_cov = ctx->d_mem = ctx->d_port = nullptr;
  ctx->src = SRC_NONE;
  ctx->N = ctx->T = ctx->cycle = 0;
  ctx->device_bytes = ctx->static_bytes;
}


constexpr uint32_t kJitMaxLanes = 8;   // JIT op-lanes by default (16 when few tiles fit a CTA, see load)
constexpr uint64_t kMaxStimuli = 65535ull * 32ull;   // per context: transposes' grid.y bound

// descriptor staging buffers start after the slots, 16-byte aligned
static uint32_t desc_smem_off(const Program &G) { return (G.smem_words + 3u) & ~3u; }

// ------------------------------------------------------------------ load --
extern "C" int rtlsim_load(const rtlsim_ir *ir, const rtlsim_options *opt, rtlsim_ctx **out) {
  if (!out) {
    g_load_error = "NULL out";
    return RTLSIM_E_ARG;
  }
  *out = nullptr;
  rtlsim_ctx *ctx = new (std::nothrow) rtlsim_ctx();
  if (!ctx) return RTLSIM_E_NOMEM;
  if (opt) ctx->opt = *opt;
  ctx->host_only = (ctx->opt.flags & RTLSIM_F_HOST_ONLY) != 0;
  ctx->device = ctx->opt.device;
  uint32_t smem_limit = ctx->opt.smem_limit;
  if (!ctx->host_only) {
    cudaError_t e = cudaSetDevice(ctx->device);
    if (e == cudaSuccess) {
      int optin = 0;
      e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->device);
      if (!smem_limit) smem_limit = (uint32_t)optin;
      smem_limit = std::min<uint32_t>(smem_limit, (uint32_t)optin);
    }
    if (e != cudaSuccess) {
      g_load_error = std::string("CUDA device unavailable: ") + cudaGetErrorString(e);
      cudaGetLastError();
      delete ctx;
      return RTLSIM_E_CUDA;
    }
  } else if (!smem_limit) {
    smem_limit = 232448;   // sm_100 opt-in maximum (227 KB)
  }
  std::string err;
  // JIT kernels are instruction-fetch bound: fewer, longer per-warp code runs
  // and more tiles sharing them measure faster (config 3: 4 op-lanes x 4
  // tiles 0.74 ms/cycle, 8 x 2 1.08 ms, 16 x 1 3.5 ms)
  uint32_t lanes = ctx->opt.op_lanes;
  const bool dce = (ctx->opt.flags & RTLSIM_F_NO_DCE) == 0;
  const bool fold = (ctx->opt.flags & RTLSIM_F_JIT) != 0 && !getenv("RTLSIM_NO_FOLD");   // JIT-only store-with-conversion descriptors
  if (!lanes && (ctx->opt.flags & RTLSIM_F_JIT)) lanes = kJitMaxLanes;
  const bool tmem = false;   // the TMEM schedule is chosen below, after the classic one
  int rc = compile_program(ir, lanes, smem_limit / 4u, &ctx->prog, &err, dce, fold);
  if (rc == RTLSIM_OK && !ctx->opt.op_lanes && (ctx->opt.flags & RTLSIM_F_JIT) && ctx->prog.L > 1) {
    // keep the auto choice when it is smaller than the cap
    rtlsim::Program probe;
    std::string e2;
    if (compile_program(ir, 0, smem_limit / 4u, &probe, &e2, dce, fold) == RTLSIM_OK && probe.L < ctx->prog.L)
      ctx->prog = std::move(probe);
  }
  if (rc != RTLSIM_OK) {
    g_load_error = err;
    delete ctx;
    return rc;
  }
  if ((ctx->prog.MR || !ctx->prog.wports.empty()) && !(ctx->opt.flags & RTLSIM_F_JIT)) {
    // memories (ARRSEL reads, write ports) are generated code only
    g_load_error = "memories (MEMRD / write ports) need RTLSIM_F_JIT";
    delete ctx;
    return RTLSIM_E_UNSUPPORTED;
  }
  if (ctx->opt.flags & RTLSIM_F_V4) {
    // the round-1 run-based micro-op evaluator was removed (slower than the
    // JIT kernels and the descriptor interpreter on every config)
    g_load_error = "RTLSIM_F_V4: the run-based evaluator was removed";
    delete ctx;
    return RTLSIM_E_UNSUPPORTED;
  }
  const bool legacy = true;   // the descriptor interpreter: staging buffers per op-lane
  uint32_t budget_words = smem_limit / 4u;
  if ((ctx->opt.flags & RTLSIM_F_JIT) && !ctx->opt.smem_limit && !tmem &&
      (ctx->prog.smem_words + 64u) * 4u > smem_limit / 2u) {
    // JIT kernels are instruction-fetch bound: two tiles per CTA (the warps
    // of one op-lane share every fetched instruction) beat one tile with the
    // whole working set on chip (config 4: 193 vs 306 ms/cycle), so the
    // working set is budgeted to half the shared memory (long-lived values
    // spill to HBM rows)
    rtlsim::Program half;
    std::string e2;
    if (compile_program(ir, ctx->prog.L, (smem_limit / 2u - 1024u) / 4u, &half, &e2, dce, fold) == RTLSIM_OK) {
      ctx->prog = std::move(half);
      budget_words = (smem_limit / 2u - 1024u) / 4u;
    }
  }
  if ((ctx->opt.flags & RTLSIM_F_JIT) && !ctx->opt.op_lanes && !tmem && ctx->prog.L == kJitMaxLanes) {
    // Occupancy: as many warps per SM as a 1024-thread CTA holds. K tiles fit
    // the shared memory; more op-lanes per tile fill the CTA when K is small
    // (measured round 2, profiles/r02_sweep_*.log: config 4 (K = 2) 4 / 8 /
    // 16 op-lanes 145 / 79 / 75 ms per cycle; config 3 (K = 4) 8 op-lanes
    // 1.22 ms vs 16 x 2 tiles 2.19 ms)
    const uint32_t K = std::max<uint32_t>(
        1u, std::min<uint32_t>(jit_default_tiles(), smem_limit / std::max<uint32_t>(jit_tile_bytes(ctx->prog), 1u)));
    // (r2 sweep, profiles/r02_i_probe.log / r02_j_probe.log, config 4 at two
    // tiles: 10 / 12 / 13 / 14 / 16 op-lanes 73.6 / 72.6 / 73.0 / 72.4 / 75.5 ms)
    const uint32_t want = K == 1 ? 16u : K == 2 ? 14u : std::min<uint32_t>(16u, 32u / K);
    if (want > ctx->prog.L) {
      rtlsim::Program wide;
      std::string e2;
      if (compile_program(ir, want, budget_words, &wide, &e2, dce, fold) == RTLSIM_OK &&
          wide.smem_words <= ctx->prog.smem_words)
        ctx->prog = std::move(wide);
    }
  }
  // (r2) TMEM schedule (JIT): U32 values computed by ops live in tensor
  // memory, four tiles per CTA (one per TMEM lane quarter / SMSP), up to 8
  // op-lanes. The JIT kernels are instruction-fetch bound:
  // four warps sharing each fetched instruction instead of two measured
  // config 4 at 55.6 vs 76.2 ms/cycle; designs whose classic working set
  // already fits four tiles gain nothing (config 3: 1.59 vs 1.47). Auto:
  // when fewer than four classic tiles fit; RTLSIM_JIT_TMEM=1 / 0 forces.
  if ((ctx->opt.flags & RTLSIM_F_JIT) && !ctx->opt.smem_limit && jit_tmem_mode() != 0) {
    const bool want = jit_tmem_mode() == 1 || jit_tile_bytes(ctx->prog) * 4u + 256u > smem_limit;
    if (want) {
      rtlsim::Program tp;
      std::string e2;
      const uint32_t tl = std::min<uint32_t>(ctx->opt.op_lanes ? ctx->opt.op_lanes : 8u, 8u);
      // RTLSIM_JIT_TMEM_SMEM_KB: CTA shared-memory budget (the rest of the
      // 256 KB is L1, where register spills land)
      uint32_t cta = smem_limit;
      if (const char *e = getenv("RTLSIM_JIT_TMEM_SMEM_KB")) cta = std::min<uint32_t>(cta, 1024u * (uint32_t)atoi(e));
      if (compile_program(ir, tl, (cta - 256u) / 16u, &tp, &e2, dce, fold, 512u) == RTLSIM_OK &&
          tp.tmem_cols > 0 && jit_tile_bytes(tp) * 4u + 256u <= smem_limit)
        ctx->prog = std::move(tp);
    }
  }
  // bytes: slots and, for the interpreter, one 512-byte descriptor staging
  // buffer per op-lane
  auto final_bytes = [&](const Program &P) {
    uint32_t w = (P.smem_words + 3u) & ~3u;
    return (legacy ? ((w + 3u) & ~3u) * 4u + P.L * 512u : w * 4u);
  };
  if (final_bytes(ctx->prog) > smem_limit) {
    // these come out of the same budget: recompile the slot area against
    // what is left
    const uint32_t L = ctx->prog.L, reserve = (legacy ? L * 512u : 0u) + 160u;
    if (smem_limit > reserve) {
      rtlsim::Program again;
      std::string e2;
      rc = compile_program(ir, L, (smem_limit - reserve) / 4u, &again, &e2, dce, fold);
      if (rc != RTLSIM_OK) {
        g_load_error = e2;
        delete ctx;
        return rc;
      }
      ctx->prog = std::move(again);
    }
  }
  Program &G = ctx->prog;
  // interpreter: slots + one 512-byte descriptor staging buffer per op-lane warp
  ctx->smem_bytes = legacy ? desc_smem_off(G) * 4u + G.L * 512u : G.smem_words * 4u;
  if (ctx->smem_bytes > smem_limit) {
    g_load_error = "per-tile working set of " + std::to_string(ctx->smem_bytes) +
                   " bytes (with descriptor buffers) exceeds the shared-memory limit";
    delete ctx;
    return RTLSIM_E_NOMEM;
  }
  if (ctx->opt.chunk_cycles) ctx->Tc = ctx->opt.chunk_cycles;
  auto jit_setup = [&](int device) -> int {
    Dl_info info;
    std::string dir = ".";
    if (dladdr((void *)&rtlsim_load, &info) && info.dli_fname) {
      dir = info.dli_fname;
      dir = dir.substr(0, dir.find_last_of('/'));
    }
    ctx->jit_smem = std::max<uint32_t>(jit_tile_bytes(G), 16u);
    ctx->jit_rt_path = dir + "/jit_rt.ptx";
    ctx->jit_smem_cap = std::min<uint32_t>(ctx->jit_smem * jit_default_tiles(), smem_limit);
    // device contexts compile at the first run, specialised for the bound
    // N_pad (jit_ensure); RTLSIM_JIT_GENERIC=1 keeps the N-generic kernels,
    // built here. Host-only: generic, or RTLSIM_JIT_NSPEC=<N_pad> (inspection)
    uint32_t nspec = 0;
    if (device < 0 && getenv("RTLSIM_JIT_NSPEC")) nspec = (uint32_t)atoi(getenv("RTLSIM_JIT_NSPEC"));
    if (device >= 0 && jit_specialise()) return RTLSIM_OK;
    std::string jerr;
    int jr = jit_build(G, ctx->jit_rt_path, ctx->jit_smem_cap, device, &ctx->jit, &jerr, false, nspec);
    if (jr == RTLSIM_OK && (ctx->opt.flags & RTLSIM_F_DIGEST))
      jr = jit_build(G, ctx->jit_rt_path, ctx->jit_smem_cap, device, &ctx->jit_dig, &jerr, true, nspec);
    if (jr != RTLSIM_OK) g_load_error = "JIT: " + jerr;
    return jr;
  };
  if (ctx->host_only) {
    if (ctx->opt.flags & RTLSIM_F_JIT) {
      int jr = jit_setup(-1);   // generate + compile (no device needed)
      if (jr != RTLSIM_OK) {
        delete ctx;
        return jr;
      }
    }
    *out = ctx;
    return RTLSIM_OK;
  }
  // device-side static data
  auto up = [&](void **dst, const void *src, size_t bytes) -> cudaError_t {
    cudaError_t e = dalloc(ctx, dst, std::max<size_t>(bytes, 16), false);
    if (e != cudaSuccess || !bytes) return e;
    return cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice);
  };
  std::vector<RegWord> regmap(G.RW);
  for (const RegInfo &ri : G.regs)
    for (uint32_t t = 0; t < (ri.cls == CLS_U32 ? nwords(ri.width) : 1u); t++)
      regmap[ri.word + t] = RegWord{ri.cls, ri.row + t};
  cudaError_t e = cudaSuccess;
  // the evaluator prefetches descriptor chunks of 16 past the end: pad
  std::vector<Desc> padded(G.desc);
  padded.resize(G.desc.size() + 32, Desc{});   // chunk prefetch reads up to 32 past any start
  if (e == cudaSuccess) e = up((void **)&ctx->d_desc, padded.data(), padded.size() * sizeof(Desc));
  if (e == cudaSuccess) e = up((void **)&ctx->d_bitdesc, G.bitdesc.data(), G.bitdesc.size() * sizeof(BitDesc));
  if (e == cudaSuccess) e = up((void **)&ctx->d_bitptr, G.bit_ptr.data(), G.bit_ptr.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_stepwait, G.step_wait.data(), G.step_wait.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_wide, G.wide.data(), G.wide.size() * sizeof(WideRec));
  if (e == cudaSuccess) e = up((void **)&ctx->d_inmap, G.in_map.data(), G.in_map.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_step, G.step_ptr.data(), G.step_ptr.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_consts, G.const_pool.data(), G.const_pool.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_mask, G.in_mask.data(), G.in_mask.size() * 4);
  if (e == cudaSuccess) e = up((void **)&ctx->d_regmap, regmap.data(), regmap.size() * sizeof(RegWord));
  if (e == cudaSuccess) e = up((void **)&ctx->d_reginit, G.reg_init.data(), G.reg_init.size() * 4);
  if (!G.wports.empty() || G.MR) {
    std::vector<MemPortDev> mp;
    for (const Program::WPort &w : G.wports)
      mp.push_back(MemPortDev{G.mem_row0[w.mem], G.mem_depth[w.mem], G.mem_width[w.mem], w.addr_word, w.data_word,
                              w.data_width, w.en_word, w.en_width});
    if (e == cudaSuccess) e = up((void **)&ctx->d_ports, mp.data(), mp.size() * sizeof(MemPortDev));
    if (e == cudaSuccess) e = up((void **)&ctx->d_meminit, G.mem_init.data(), G.mem_init.size() * 4);
  }
  if (e == cudaSuccess) e = eval_set_smem(std::max<uint32_t>(ctx->smem_bytes, 1024));
  if (e == cudaSuccess) {
    if (ctx->opt.cuda_stream) {
      ctx->st = (cudaStream_t)ctx->opt.cuda_stream;
    } else {
      e = cudaStreamCreateWithFlags(&ctx->st, cudaStreamNonBlocking);
      ctx->own_stream = true;
    }
  }
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->st_h2d, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->st_d2h, cudaStreamNonBlocking);
  for (int b = 0; b < 2 && e == cudaSuccess; b++) {
    e = cudaEventCreateWithFlags(&ctx->ev_in_ready[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_comp_done[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_drain_done[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_h2d_copied[b], cudaEventDisableTiming);
  }
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->ev_start, cudaEventDisableTiming);
  if (e != cudaSuccess) {
    g_load_error = std::string("CUDA error during load: ") + cudaGetErrorString(e);
    cudaGetLastError();
    rtlsim_free(ctx);
    return e == cudaErrorMemoryAllocation ? RTLSIM_E_NOMEM : RTLSIM_E_CUDA;
  }
  if (ctx->opt.flags & RTLSIM_F_JIT) {
    int jr = jit_setup(ctx->device);
    if (jr != RTLSIM_OK) {
      rtlsim_free(ctx);
      return jr;
    }
  }
  ctx->static_bytes = ctx->device_bytes;
  *out = ctx;
  return RTLSIM_OK;
}

// ------------------------------------------------------------------ bind --
static int alloc_arena(rtlsim_ctx *ctx, Arena *a, const uint32_t rows[4]) {
  const size_t N = ctx->N_pad;
  CK(dalloc(ctx, (void **)&a->bit, (size_t)rows[CLS_BIT] * (N / 32) * 4, true));
  CK(dalloc(ctx, (void **)&a->u8, (size_t)rows[CLS_U8] * N, true));
  CK(dalloc(ctx, (void **)&a->u16, (size_t)rows[CLS_U16] * N * 2, true));
  CK(dalloc(ctx, (void **)&a->u32, (size_t)rows[CLS_U32] * N * 4, true));
  return RTLSIM_OK;
}

static int reset_regs(rtlsim_ctx *ctx) {
  Program &G = ctx->prog;
  if (G.MR && ctx->d_mem) {   // memories back to their initial contents
    CK(launch_mem_init(ctx->d_mem, ctx->d_meminit, G.MR, ctx->N_pad, ctx->st));
    ctx->launches++;
  }
  CK(launch_regs_import(ctx->d_reginit, 0, ctx->d_regmap, G.RW, (uint32_t)ctx->N, ctx->N_pad, ctx->state[0],
                        ctx->st));
  ctx->launches++;
  ctx->cycle = 0;
  return RTLSIM_OK;
}

static int bind_common(rtlsim_ctx *ctx, uint64_t N, uint64_t T) {
  if (!ctx) return RTLSIM_E_ARG;
  if (ctx->failed || ctx->host_only) return arg_fail(ctx, RTLSIM_E_STATE, ctx->failed ? ctx->err : "host-only ctx");
  // the N2 / N3 / digest transposes put the 32-stimulus tiles in grid.y
  // (<= 65535 blocks): N <= 65535 * 32 stimuli per context (per GPU shard)
  if (N == 0 || N > kMaxStimuli) return arg_fail(ctx, RTLSIM_E_ARG, "N out of range (1..2097120 per context)");
  CK(cudaSetDevice(ctx->device));
  CK(cudaStreamSynchronize(ctx->st));
  CK(cudaStreamSynchronize(ctx->st_h2d));
  CK(cudaStreamSynchronize(ctx->st_d2h));
  free_binding(ctx);
  ctx->N = N;
  ctx->T = T;
  // (r2) TMEM kernels run exactly four tiles per CTA: N_pad in 128s
  const uint64_t padq = ctx->prog.tmem_cols ? 128u : 32u;
  ctx->N_pad = (uint32_t)((N + padq - 1) / padq * padq);
  Program &G = ctx->prog;
  ctx->Tc = ctx->opt.chunk_cycles ? ctx->opt.chunk_cycles : 64;
  if (T) ctx->Tc = (uint32_t)std::min<uint64_t>(ctx->Tc, T);
  ctx->Tc = std::max<uint32_t>(ctx->Tc, 1);
  int rc;
  for (int b = 0; b < 2; b++)
    if ((rc = alloc_arena(ctx, &ctx->state[b], G.rows)) != RTLSIM_OK) return rc;
  if ((rc = alloc_arena(ctx, &ctx->xnet, G.xrows)) != RTLSIM_OK) return rc;
  if (G.MR) CK(dalloc(ctx, (void **)&ctx->d_mem, (size_t)G.MR * ctx->N_pad * 4, true));
  if (G.PW) CK(dalloc(ctx, (void **)&ctx->d_port, (size_t)G.PW * ctx->N_pad * 4, true));
  if ((ctx->opt.flags & RTLSIM_F_COVERAGE) && G.RW) {
    CK(dalloc(ctx, (void **)&ctx->d_cov, (size_t)G.RW * 4, true));
    CK(cudaMemsetAsync(ctx->d_cov, 0, (size_t)G.RW * 4, ctx->st));
  }
  const size_t NP = ctx->N_pad, Tc = ctx->Tc;
  ctx->in_stride.s[CLS_BIT] = (uint64_t)G.in_rows[CLS_BIT] * (NP / 32);
  ctx->in_stride.s[CLS_U8] = (uint64_t)G.in_rows[CLS_U8] * NP;
  ctx->in_stride.s[CLS_U16] = (uint64_t)G.in_rows[CLS_U16] * NP;
  ctx->in_stride.s[CLS_U32] = (uint64_t)G.in_rows[CLS_U32] * NP;
  for (int b = 0; b < 2; b++) {
    CK(dalloc(ctx, (void **)&ctx->d_in[b].bit, std::max<size_t>(Tc * ctx->in_stride.s[CLS_BIT] * 4, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_in[b].u8, std::max<size_t>(Tc * ctx->in_stride.s[CLS_U8], 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_in[b].u16, std::max<size_t>(Tc * ctx->in_stride.s[CLS_U16] * 2, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_in[b].u32, std::max<size_t>(Tc * ctx->in_stride.s[CLS_U32] * 4, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_out[b], std::max<size_t>(Tc * G.OW * NP * 4, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_dig[b], Tc * NP * 8, true));
    ctx->ev_used[b] = false;
  }
  return reset_regs(ctx);
}

// lazily allocated staging used by host-buffer / callback runs
static int ensure_host_staging(rtlsim_ctx *ctx) {
  if (ctx->d_raw[0]) return RTLSIM_OK;
  Program &G = ctx->prog;
  const size_t N = ctx->N, Tc = ctx->Tc;
  for (int b = 0; b < 2; b++) {
    CK(dalloc(ctx, (void **)&ctx->d_raw[b], std::max<size_t>(N * Tc * G.IW * 4, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_outu[b], std::max<size_t>(N * Tc * G.OW * 4, 16), true));
    CK(dalloc(ctx, (void **)&ctx->d_digu[b], N * Tc * 8, true));
    void *p;
    CK(cudaMallocHost(&p, std::max<size_t>(N * Tc * G.IW * 4, 16)));
    ctx->host_allocs.push_back(p);
    ctx->h_in[b] = (uint32_t *)p;
    CK(cudaMallocHost(&p, std::max<size_t>(N * Tc * G.OW * 4, 16)));
    ctx->host_allocs.push_back(p);
    ctx->h_out[b] = (uint32_t *)p;
    CK(cudaMallocHost(&p, N * Tc * 8));
    ctx->host_allocs.push_back(p);
    ctx->h_dig[b] = (unsigned long long *)p;
  }
  return RTLSIM_OK;
}

extern "C" int rtlsim_bind(rtlsim_ctx *ctx, uint64_t N, uint64_t T, const uint32_t *stim) {
  if (!ctx) return RTLSIM_E_ARG;
  if (!stim && ctx->prog.IW && T) return arg_fail(ctx, RTLSIM_E_ARG, "NULL stimulus");
  int rc = bind_common(ctx, N, T);
  if (rc) return rc;
  ctx->src = SRC_HOST;
  ctx->stim = stim;
  ctx->stim_pinned = is_pinned(stim);
  return RTLSIM_OK;
}

extern "C" int rtlsim_bind_device(rtlsim_ctx *ctx, uint64_t N, uint64_t T, const uint32_t *stim_dev) {
  if (!ctx) return RTLSIM_E_ARG;
  if (!stim_dev && ctx->prog.IW && T) return arg_fail(ctx, RTLSIM_E_ARG, "NULL stimulus");
  int rc = bind_common(ctx, N, T);
  if (rc) return rc;
  ctx->src = SRC_DEVICE;
  ctx->stim = stim_dev;
  return RTLSIM_OK;
}

extern "C" int rtlsim_bind_stream(rtlsim_ctx *ctx, uint64_t N, uint64_t T, rtlsim_producer prod, void *user) {
  if (!ctx) return RTLSIM_E_ARG;
  if (!prod) return arg_fail(ctx, RTLSIM_E_ARG, "NULL producer");
  int rc = bind_common(ctx, N, T);
  if (rc) return rc;
  ctx->src = SRC_PRODUCER;
  ctx->prod = prod;
  ctx->prod_user = user;
  return RTLSIM_OK;
}

// ------------------------------------------------------------------- run --
static EvalParams eval_params(rtlsim_ctx *ctx, int b, uint64_t cycle0, uint32_t nc, bool digest) {
  Program &G = ctx->prog;
  EvalParams p{};
  p.desc = ctx->d_desc;
  p.bitdesc = ctx->d_bitdesc;
  p.bit_ptr = ctx->d_bitptr;
  p.step_wait = ctx->d_stepwait;
  p.wide = ctx->d_wide;
  p.step_ptr = ctx->d_step;
  p.step_begin = 0;
  p.step_end = G.n_steps;
  p.L = G.L;
  p.n_cycles = nc;
  p.cycle0 = cycle0;
  p.N_pad = ctx->N_pad;
  p.IW = G.IW;
  p.OW = G.OW;
  p.state[0] = ctx->state[0];
  p.state[1] = ctx->state[1];
  p.xnet = ctx->xnet;
  p.in = ctx->d_in[b];
  for (int k = 0; k < 4; k++) p.in_stride[k] = ctx->in_stride.s[k];
  p.desc_smem_off = desc_smem_off(G);
  p.out = ctx->d_out[b];
  p.consts = ctx->d_consts;
  p.digest = digest ? ctx->d_dig[b] : nullptr;
  return p;
}

// JIT kernels for the bound N_pad (specialised unless RTLSIM_JIT_GENERIC):
// built on first use and whenever a rebind changed N_pad; check-mode
// (digest) kernels separately, on first use
static int jit_ensure(rtlsim_ctx *ctx, bool dig) {
  JitKernels &K = dig ? ctx->jit_dig : ctx->jit;
  const uint32_t want = jit_specialise() ? ctx->N_pad : 0;
  if (!K.kern.empty() && K.nspec == want) return RTLSIM_OK;
  CK(cudaStreamSynchronize(ctx->st));
  jit_free(&K);
  std::string jerr;
  int jr = jit_build(ctx->prog, ctx->jit_rt_path, ctx->jit_smem_cap, ctx->device, &K, &jerr, dig, want);
  if (jr != RTLSIM_OK) {
    ctx->failed = true;
    ctx->err = std::string(dig ? "JIT (digest variant): " : "JIT: ") + jerr;
    return jr;
  }
  return RTLSIM_OK;
}

// JIT: tiles per CTA — as many as the shared memory holds (up to the count
// the kernels were compiled for) that divide the tile count; env override
// RTLSIM_JIT_TPC for measurements
static uint32_t jit_tile_smem(rtlsim_ctx *ctx, const JitKernels &JK, uint32_t q) {
  return q < JK.tile_bytes.size() && JK.tile_bytes[q] ? JK.tile_bytes[q] : ctx->jit_smem;
}
static uint32_t jit_tiles_per_cta(rtlsim_ctx *ctx, const JitKernels &JK, uint32_t q) {
  const uint32_t tiles = ctx->N_pad / 32u;
  int optin = 232448;
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->device);
  // the kernel set being launched (the check-mode variant may have been built
  // with another RTLSIM_JIT_TMAX than the plain one): its .maxntid bound; the
  // partition's own shared memory per tile (compacted kernels differ)
  if (ctx->prog.tmem_cols) return 4u;   // one tile per TMEM lane quarter
  uint32_t m = std::min<uint32_t>(JK.tmax, ((uint32_t)optin - 16u) / std::max<uint32_t>(jit_tile_smem(ctx, JK, q), 1u));
  if (const char *e = getenv("RTLSIM_JIT_TPC")) m = std::min<uint32_t>(m, (uint32_t)atoi(e));
  m = std::max<uint32_t>(m, 1u);
  // small batches (config 2: 128 tiles): fewer tiles per CTA so that every
  // SM gets a CTA, rather than K tiles on a quarter of the SMs
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, ctx->device);
  while (m > 1 && tiles / m < (uint32_t)sms) m--;
  while (m > 1 && tiles % m) m--;
  return m;
}

static cudaError_t evaluator(rtlsim_ctx *ctx, const EvalParams &p, cudaStream_t st) {
  return launch_eval(p, ctx->smem_bytes, st);
}

static cudaError_t get_event(rtlsim_ctx *ctx, cudaEvent_t *e) {
  if (!ctx->event_pool.empty()) {
    *e = ctx->event_pool.back();
    ctx->event_pool.pop_back();
    return cudaSuccess;
  }
  return cudaEventCreate(e);
}

// fold completed timing events into the totals (blocking on them)
static int fold_timing(rtlsim_ctx *ctx) {
  for (auto &t : ctx->timed_pending) {
    CK(cudaEventSynchronize(t.b));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, t.a, t.b));
    ctx->eval_ms += ms;
    ctx->eval_launches++;
    ctx->eval_stim_cycles += t.stim_cycles;
    ctx->event_pool.push_back(t.a);
    ctx->event_pool.push_back(t.b);
  }
  ctx->timed_pending.clear();
  return RTLSIM_OK;
}

// simulate chunk (cycle0, nc) from d_in[b] into d_out[b] / d_dig[b] on ctx->st
static int launch_chunk(rtlsim_ctx *ctx, int b, uint64_t cycle0, uint32_t nc, bool digest) {
  Program &G = ctx->prog;
  if (digest) CK(cudaMemsetAsync(ctx->d_dig[b], 0, (size_t)nc * ctx->N_pad * 8, ctx->st));
  if (G.n_steps == 0) return RTLSIM_OK;
  const bool timing = (ctx->opt.flags & RTLSIM_F_TIMING) != 0;
  rtlsim_ctx::Timed tm{nullptr, nullptr, (uint64_t)nc * ctx->N};
  if (timing) {
    CK(get_event(ctx, &tm.a));
    CK(get_event(ctx, &tm.b));
    CK(cudaEventRecord(tm.a, ctx->st));
  }
  // the fused interpreter runs a whole chunk in one launch; coverage needs a
  // cycle boundary, so it uses the per-(cycle, partition) graph instead
  if (!(ctx->opt.flags & (RTLSIM_F_GRAPH | RTLSIM_F_JIT | RTLSIM_F_STREAM | RTLSIM_F_COVERAGE))) {
    EvalParams p = eval_params(ctx, b, cycle0, nc, digest);
    CK(evaluator(ctx, p, ctx->st));
    ctx->launches++;
    if (timing) {
      CK(cudaEventRecord(tm.b, ctx->st));
      ctx->timed_pending.push_back(tm);
    }
    return RTLSIM_OK;
  }
  const bool jit = (ctx->opt.flags & RTLSIM_F_JIT) != 0;
  if (jit) {   // normally built by run_impl already
    int jr = jit_ensure(ctx, digest);
    if (jr != RTLSIM_OK) return jr;
  }
  const JitKernels &JK = digest ? ctx->jit_dig : ctx->jit;
  // M1 persistent mode: a single-partition design with no
  // per-cycle sink kernels (memory ports, coverage) runs a whole chunk of
  // cycles in one launch per CTA; RTLSIM_M1=0 keeps one launch per cycle
  const bool m1 = jit && G.part_steps.size() == 2 && G.wports.empty() && !ctx->d_cov &&
                  !(ctx->opt.flags & RTLSIM_F_STREAM) && !(getenv("RTLSIM_M1") && atoi(getenv("RTLSIM_M1")) == 0);
  // Tc x P per-(cycle, partition) kernel nodes (graph / JIT / stream modes).
  // Captured graphs (RTLSIM_DAG, default on) get the partition DAG's edges
  // instead of a chain: within a cycle a partition waits only for the
  // partitions whose nets it reads (and spilling partitions for each other),
  // so independent partitions overlap (partitioning "maximizes
  // the kernel concurrency of the induced CUDA graph"); every cycle still
  // starts after the whole previous cycle (registers and nets are reused).
  // Default: on when a partition launch is at most 4 waves of CTAs (its tail
  // is a large share; config 3: 1.22 -> 1.12 ms/cycle), off for long
  // launches (config 4, 6.9 waves: 75.6 -> 84.1 ms/cycle with it, two
  // partitions' code streams compete for instruction fetch);
  // profiles/r02_f_probe.log
  bool dag_env = !getenv("RTLSIM_DAG") || atoi(getenv("RTLSIM_DAG")) != 0;
  if (!getenv("RTLSIM_DAG") && jit) {
    uint32_t ctas = 0;
    for (uint32_t q = 0; q + 1 < G.part_steps.size(); q++)
      if (q < JK.kern.size() && JK.kern[q]) ctas = std::max(ctas, ctx->N_pad / 32u / jit_tiles_per_cta(ctx, JK, q));
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, ctx->device);
    dag_env = ctas <= 4u * (uint32_t)sms;
  }
  auto issue = [&](cudaStream_t cap) -> cudaError_t {
    const uint32_t NP = (uint32_t)G.part_steps.size() - 1;
    const bool dag = dag_env && cap != ctx->st && NP > 1;
    if (dag && ctx->dag_streams.empty()) {
      for (int i = 0; i < 8; i++) {
        cudaStream_t x;
        cudaError_t e = cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking);
        if (e != cudaSuccess) return e;
        ctx->dag_streams.push_back(x);
      }
      cudaError_t e = cudaEventCreateWithFlags(&ctx->dag_fork, cudaEventDisableTiming);
      if (e != cudaSuccess) return e;
    }
    while (dag && ctx->dag_events.size() < NP) {
      cudaEvent_t x;
      cudaError_t e = cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
      if (e != cudaSuccess) return e;
      ctx->dag_events.push_back(x);
    }
    for (uint32_t c = 0; c < nc; c += (m1 ? nc : 1)) {
      if (dag) {
        cudaError_t e = cudaEventRecord(ctx->dag_fork, cap);
        if (e != cudaSuccess) return e;
      }
      std::vector<char> issued(NP, 0);
      for (uint32_t q = 0; q < NP; q++) {
        if (G.part_steps[q] == G.part_steps[q + 1]) continue;
        cudaError_t e;
        cudaStream_t sq = cap;
        if (dag) {
          sq = ctx->dag_streams[q % ctx->dag_streams.size()];
          if ((e = cudaStreamWaitEvent(sq, ctx->dag_fork, 0)) != cudaSuccess) return e;
          for (uint32_t p : G.part_dep[q])
            if (issued[p] && (e = cudaStreamWaitEvent(sq, ctx->dag_events[p], 0)) != cudaSuccess) return e;
        }
        if (jit) {
          if (!JK.kern[q]) continue;
          const uint32_t par = (uint32_t)(((cycle0 & 1ull) + c) & 1ull);
          JitParams jp{};
          const Arena *ar[3] = {&ctx->state[par], &ctx->state[par ^ 1u], &ctx->xnet};
          uint64_t *dst[3] = {jp.cur, jp.nxt, jp.xnet};
          for (int t = 0; t < 3; t++) {
            dst[t][0] = (uint64_t)ar[t]->bit; dst[t][1] = (uint64_t)ar[t]->u8;
            dst[t][2] = (uint64_t)ar[t]->u16; dst[t][3] = (uint64_t)ar[t]->u32;
          }
          jp.in[0] = (uint64_t)(ctx->d_in[b].bit + (size_t)c * ctx->in_stride.s[CLS_BIT]);
          jp.in[1] = (uint64_t)(ctx->d_in[b].u8 + (size_t)c * ctx->in_stride.s[CLS_U8]);
          jp.in[2] = (uint64_t)(ctx->d_in[b].u16 + (size_t)c * ctx->in_stride.s[CLS_U16]);
          jp.in[3] = (uint64_t)(ctx->d_in[b].u32 + (size_t)c * ctx->in_stride.s[CLS_U32]);
          jp.out = (uint64_t)(ctx->d_out[b] + (size_t)c * G.OW * ctx->N_pad);
          jp.digest = digest ? (uint64_t)(ctx->d_dig[b] + (size_t)c * ctx->N_pad) : 0;
          jp.wide = JK.d_wide ? (uint64_t)(JK.d_wide + JK.wide_base[q]) : (uint64_t)ctx->d_wide;
          jp.N = ctx->N_pad;
          jp.bittab = JK.d_bittab ? (uint64_t)(JK.d_bittab + 4ull * JK.bit_base[q]) : 0;
          jp.mem = (uint64_t)ctx->d_mem;
          jp.port = (uint64_t)ctx->d_port;
          jp.nc = m1 ? nc : 1;
          jp.in_step[0] = (uint64_t)ctx->in_stride.s[CLS_BIT] * 4;
          jp.in_step[1] = (uint64_t)ctx->in_stride.s[CLS_U8];
          jp.in_step[2] = (uint64_t)ctx->in_stride.s[CLS_U16] * 2;
          jp.in_step[3] = (uint64_t)ctx->in_stride.s[CLS_U32] * 4;
          jp.out_step = (uint64_t)G.OW * ctx->N_pad * 4;
          jp.dig_step = (uint64_t)ctx->N_pad * 8;
          jp.tpc = jit_tiles_per_cta(ctx, JK, q);
          void *args[] = {&jp};
          e = cudaLaunchKernel((const void *)JK.kern[q], dim3(ctx->N_pad / 32u / jp.tpc),
                               dim3(32u * G.L * jp.tpc), args, jit_tile_smem(ctx, JK, q) * jp.tpc + 32u, sq);
        } else {
          EvalParams p = eval_params(ctx, b, (cycle0 & 1ull) + c, 1, digest);
          p.step_begin = G.part_steps[q];
          p.step_end = G.part_steps[q + 1];
          p.in.bit = ctx->d_in[b].bit + (size_t)c * ctx->in_stride.s[CLS_BIT];
          p.in.u8 = ctx->d_in[b].u8 + (size_t)c * ctx->in_stride.s[CLS_U8];
          p.in.u16 = ctx->d_in[b].u16 + (size_t)c * ctx->in_stride.s[CLS_U16];
          p.in.u32 = ctx->d_in[b].u32 + (size_t)c * ctx->in_stride.s[CLS_U32];
          p.out = ctx->d_out[b] + (size_t)c * G.OW * ctx->N_pad;
          if (digest) p.digest = ctx->d_dig[b] + (size_t)c * ctx->N_pad;
          e = evaluator(ctx, p, sq);
        }
        if (e != cudaSuccess) return e;
        if (dag) {
          if ((e = cudaEventRecord(ctx->dag_events[q], sq)) != cudaSuccess) return e;
          issued[q] = 1;
        }
      }
      if (dag)   // join: the cycle's sinks (memory ports, coverage) and the next cycle follow every partition
        for (uint32_t q = 0; q < NP; q++)
          if (issued[q]) {
            cudaError_t e = cudaStreamWaitEvent(cap, ctx->dag_events[q], 0);
            if (e != cudaSuccess) return e;
          }
      if (!G.wports.empty()) {   // memory write ports at the clock edge, after every partition
        cudaError_t e = launch_mem_commit(ctx->d_mem, ctx->d_port, ctx->d_ports, (uint32_t)G.wports.size(),
                                          (uint32_t)ctx->N, ctx->N_pad, cap);
        if (e != cudaSuccess) return e;
      }
      if (ctx->d_cov) {   // N5: toggles of this cycle's register update
        const uint32_t par = (uint32_t)(((cycle0 & 1ull) + c) & 1ull);
        cudaError_t e = launch_toggle_coverage(ctx->state[par], ctx->state[par ^ 1u], ctx->d_regmap, G.RW,
                                               (uint32_t)ctx->N, ctx->N_pad, ctx->d_cov, cap);
        if (e != cudaSuccess) return e;
      }
    }
    return cudaSuccess;
  };
  if (ctx->opt.flags & RTLSIM_F_STREAM) {
    // the paper's stream-based baseline (Table 4): the same per-(cycle,
    // partition) launches issued one by one every chunk, no graph
    CK(issue(ctx->st));
    ctx->launches += m1 ? 1 : (uint64_t)nc * (G.part_steps.size() - 1 + (ctx->d_cov ? 1 : 0) + (G.wports.empty() ? 0 : 1));
    if (timing) {
      CK(cudaEventRecord(tm.b, ctx->st));
      ctx->timed_pending.push_back(tm);
    }
    return RTLSIM_OK;
  }
  // graph mode (and JIT mode): captured once per (buffer, parity, nc, digest)
  // and replayed
  const uint64_t key = ((uint64_t)nc << 8) | ((uint64_t)b << 2) | ((cycle0 & 1ull) << 1) | (digest ? 1u : 0u);
  auto it = ctx->graphs.find(key);
  if (it == ctx->graphs.end()) {
    cudaStream_t cap;
    CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
    CK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
    cudaError_t e = issue(cap);
    cudaGraph_t g;
    cudaError_t e2 = cudaStreamEndCapture(cap, &g);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "graph capture", __LINE__);
    CK(e2);
    cudaGraphExec_t ge;
    CK(cudaGraphInstantiate(&ge, g, 0));
    CK(cudaGraphDestroy(g));
    CK(cudaStreamDestroy(cap));
    it = ctx->graphs.emplace(key, ge).first;
  }
  CK(cudaGraphLaunch(it->second, ctx->st));
  ctx->launches += m1 ? 1 : (uint64_t)nc * (G.part_steps.size() - 1 + (ctx->d_cov ? 1 : 0) + (G.wports.empty() ? 0 : 1));
  if (timing) {
    CK(cudaEventRecord(tm.b, ctx->st));
    ctx->timed_pending.push_back(tm);
  }
  return RTLSIM_OK;
}

static int run_impl(rtlsim_ctx *ctx, uint64_t cycles, const Dest &dst, bool digest) {
  if (!ctx) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "run before bind");
  if (ctx->cycle + cycles > ctx->T) return arg_fail(ctx, RTLSIM_E_RANGE, "cycles beyond the bound stimulus");
  if (cycles == 0) return RTLSIM_OK;
  Program &G = ctx->prog;
  CK(cudaSetDevice(ctx->device));
  const bool host_side = ctx->src != SRC_DEVICE || dst.out_host || dst.dig_host || dst.cons;
  if (host_side) {
    int rc = ensure_host_staging(ctx);
    if (rc) return rc;
  }
  if (ctx->opt.flags & RTLSIM_F_JIT) {
    int rc = jit_ensure(ctx, digest);
    if (rc) return rc;
  }
  const bool serial = (ctx->opt.flags & RTLSIM_F_NO_PIPELINE) != 0;
  const uint32_t N = (uint32_t)ctx->N, NP = ctx->N_pad, IW = G.IW, OW = G.OW;
  const bool out_pinned = dst.out_host && is_pinned(dst.out_host);
  const bool dig_pinned = dst.dig_host && is_pinned(dst.dig_host);
  // side streams start after everything already queued on the compute stream
  CK(cudaEventRecord(ctx->ev_start, ctx->st));
  CK(cudaStreamWaitEvent(ctx->st_h2d, ctx->ev_start, 0));
  CK(cudaStreamWaitEvent(ctx->st_d2h, ctx->ev_start, 0));

  const uint64_t nchunks = (cycles + ctx->Tc - 1) / ctx->Tc;
  std::vector<uint32_t> nc_of(nchunks);
  // A producer / consumer abort ends the run after the chunks already
  // simulated: the work queued for them completes, and the cycle cursor and
  // the register state stay consistent at the end of the last simulated
  // chunk (which can be one chunk past the one a consumer refused).
  uint64_t simulated = 0;
  auto aborted = [&](const char *why) -> int {
    cudaStreamSynchronize(ctx->st_h2d);
    cudaStreamSynchronize(ctx->st);
    cudaStreamSynchronize(ctx->st_d2h);
    ctx->cycle += simulated;
    return arg_fail(ctx, RTLSIM_E_ARG, why);
  };
  // host-side completion of chunk k (pageable outputs / consumer)
  auto finish_host = [&](uint64_t k) -> int {
    const int b = (int)(k & 1);
    const uint64_t c0 = k * ctx->Tc;
    const uint32_t nc = nc_of[k];
    if (!((dst.out_host && !out_pinned) || (dst.dig_host && !dig_pinned) || dst.cons)) return RTLSIM_OK;
    CK(cudaEventSynchronize(ctx->ev_drain_done[b]));
    if (dst.out_host && !out_pinned)
      for (uint64_t s = 0; s < N; s++)
        memcpy(dst.out_host + (s * dst.cycles + c0) * OW, ctx->h_out[b] + s * (uint64_t)nc * OW,
               (size_t)nc * OW * 4);
    if (dst.dig_host && !dig_pinned)
      for (uint64_t s = 0; s < N; s++)
        memcpy(dst.dig_host + s * dst.cycles + c0, ctx->h_dig[b] + s * (uint64_t)nc, (size_t)nc * 8);
    if (dst.cons) {
      if (dst.cons(dst.user, ctx->cycle0_run + c0, nc, ctx->h_out[b], digest ? (const uint64_t *)ctx->h_dig[b] : nullptr))
        return aborted("consumer aborted");
    }
    return RTLSIM_OK;
  };
  ctx->cycle0_run = ctx->cycle;
  for (uint64_t k = 0; k < nchunks; k++) {
    const int b = (int)(k & 1);
    const uint64_t c0 = k * ctx->Tc;
    const uint32_t nc = (uint32_t)std::min<uint64_t>(ctx->Tc, cycles - c0);
    nc_of[k] = nc;
    const uint64_t abs_c = ctx->cycle + c0;
    // ---- A: stimulus chunk -> d_in[b] (side stream)
    if (ctx->ev_used[b]) CK(cudaStreamWaitEvent(ctx->st_h2d, ctx->ev_comp_done[b], 0));
    if (IW) {
      const uint32_t *src = nullptr;
      uint64_t pitch = 0;
      if (ctx->src == SRC_DEVICE) {
        src = ctx->stim + abs_c * IW;
        pitch = ctx->T * IW;
      } else {
        const uint32_t *hsrc = nullptr;
        uint64_t hpitch = 0;
        if (ctx->src == SRC_HOST && ctx->stim_pinned) {
          hsrc = ctx->stim + abs_c * IW;
          hpitch = ctx->T * IW;
        } else {
          if (ctx->ev_used[b]) CK(cudaEventSynchronize(ctx->ev_h2d_copied[b]));
          if (ctx->src == SRC_HOST) {
            for (uint64_t s = 0; s < N; s++)
              memcpy(ctx->h_in[b] + s * (uint64_t)nc * IW, ctx->stim + (s * ctx->T + abs_c) * IW,
                     (size_t)nc * IW * 4);
          } else if (ctx->prod(ctx->prod_user, abs_c, nc, ctx->h_in[b])) {
            return aborted("producer aborted");
          }
          hsrc = ctx->h_in[b];
          hpitch = (uint64_t)nc * IW;
        }
        CK(cudaMemcpy2DAsync(ctx->d_raw[b], (size_t)nc * IW * 4, hsrc, hpitch * 4, (size_t)nc * IW * 4, N,
                             cudaMemcpyHostToDevice, ctx->st_h2d));
        CK(cudaEventRecord(ctx->ev_h2d_copied[b], ctx->st_h2d));
        src = ctx->d_raw[b];
        pitch = (uint64_t)nc * IW;
      }
      CK(launch_stim_transpose(src, pitch, N, NP, nc, IW, ctx->d_mask, ctx->d_inmap, ctx->d_in[b], ctx->in_stride,
                               ctx->st_h2d));
      ctx->launches++;
    }
    CK(cudaEventRecord(ctx->ev_in_ready[b], ctx->st_h2d));
    if (serial) CK(cudaStreamSynchronize(ctx->st_h2d));
    // ---- B: simulate the chunk (compute stream)
    CK(cudaStreamWaitEvent(ctx->st, ctx->ev_in_ready[b], 0));
    if (ctx->ev_used[b]) CK(cudaStreamWaitEvent(ctx->st, ctx->ev_drain_done[b], 0));
    int rc = launch_chunk(ctx, b, abs_c, nc, digest);
    if (rc) return rc;
    simulated += nc;
    CK(cudaEventRecord(ctx->ev_comp_done[b], ctx->st));
    if (serial) CK(cudaStreamSynchronize(ctx->st));
    // ---- C: drain (side stream)
    CK(cudaStreamWaitEvent(ctx->st_d2h, ctx->ev_comp_done[b], 0));
    if (dst.out_dev) {
      CK(launch_out_transpose(ctx->d_out[b], N, NP, nc, OW, dst.out_dev + c0 * OW, dst.cycles * OW, ctx->st_d2h));
      ctx->launches++;
    }
    if (dst.dig_dev) {
      CK(launch_digest_transpose(ctx->d_dig[b], N, NP, nc, (unsigned long long *)dst.dig_dev + c0, dst.cycles,
                                 ctx->st_d2h));
      ctx->launches++;
    }
    if (dst.out_host || dst.cons) {
      CK(launch_out_transpose(ctx->d_out[b], N, NP, nc, OW, ctx->d_outu[b], (uint64_t)nc * OW, ctx->st_d2h));
      ctx->launches++;
      if (out_pinned)
        CK(cudaMemcpy2DAsync(dst.out_host + c0 * OW, dst.cycles * OW * 4, ctx->d_outu[b], (size_t)nc * OW * 4,
                             (size_t)nc * OW * 4, N, cudaMemcpyDeviceToHost, ctx->st_d2h));
      else
        CK(cudaMemcpyAsync(ctx->h_out[b], ctx->d_outu[b], (size_t)N * nc * OW * 4, cudaMemcpyDeviceToHost,
                           ctx->st_d2h));
    }
    if (dst.dig_host || (dst.cons && digest)) {
      CK(launch_digest_transpose(ctx->d_dig[b], N, NP, nc, ctx->d_digu[b], nc, ctx->st_d2h));
      ctx->launches++;
      if (dig_pinned)
        CK(cudaMemcpy2DAsync(dst.dig_host + c0, dst.cycles * 8, ctx->d_digu[b], (size_t)nc * 8, (size_t)nc * 8, N,
                             cudaMemcpyDeviceToHost, ctx->st_d2h));
      else
        CK(cudaMemcpyAsync(ctx->h_dig[b], ctx->d_digu[b], (size_t)N * nc * 8, cudaMemcpyDeviceToHost,
                           ctx->st_d2h));
    }
    CK(cudaEventRecord(ctx->ev_drain_done[b], ctx->st_d2h));
    ctx->ev_used[b] = true;
    if (serial) CK(cudaStreamSynchronize(ctx->st_d2h));
    if (k >= 1) {
      rc = finish_host(k - 1);
      if (rc) return rc;
    }
  }
  int rc = finish_host(nchunks - 1);
  if (rc) return rc;
  // join the side streams into the compute stream
  CK(cudaEventRecord(ctx->ev_start, ctx->st_d2h));
  CK(cudaStreamWaitEvent(ctx->st, ctx->ev_start, 0));
  ctx->cycle += cycles;
  return RTLSIM_OK;
}

static int export_regs(rtlsim_ctx *ctx, uint32_t *regs_host) {
  Program &G = ctx->prog;
  if (!G.RW) return RTLSIM_OK;
  uint32_t *tmp = nullptr;
  CK(cudaMallocAsync((void **)&tmp, (size_t)ctx->N * G.RW * 4, ctx->st));
  CK(launch_regs_export(ctx->state[ctx->cycle & 1], ctx->d_regmap, G.RW, (uint32_t)ctx->N, ctx->N_pad, tmp,
                        ctx->st));
  ctx->launches++;
  CK(cudaMemcpyAsync(regs_host, tmp, (size_t)ctx->N * G.RW * 4, cudaMemcpyDeviceToHost, ctx->st));
  CK(cudaFreeAsync(tmp, ctx->st));
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_run(rtlsim_ctx *ctx, uint64_t cycles, uint32_t *out, uint32_t *regs, uint64_t *digest) {
  if (!ctx) return RTLSIM_E_ARG;
  Dest d;
  d.out_host = out;
  d.dig_host = digest;
  d.cycles = cycles;
  int rc = run_impl(ctx, cycles, d, digest != nullptr || (ctx->opt.flags & RTLSIM_F_DIGEST));
  if (rc) return rc;
  if (regs) {
    rc = export_regs(ctx, regs);
    if (rc) return rc;
  }
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_run_device(rtlsim_ctx *ctx, uint64_t cycles, uint32_t *out_dev, uint64_t *digest_dev) {
  if (!ctx) return RTLSIM_E_ARG;
  Dest d;
  d.out_dev = out_dev;
  d.dig_dev = digest_dev;
  d.cycles = cycles;
  return run_impl(ctx, cycles, d, digest_dev != nullptr);
}

extern "C" int rtlsim_run_stream(rtlsim_ctx *ctx, uint64_t cycles, rtlsim_consumer cons, void *user) {
  if (!ctx) return RTLSIM_E_ARG;
  if (!cons) return arg_fail(ctx, RTLSIM_E_ARG, "NULL consumer");
  Dest d;
  d.cons = cons;
  d.user = user;
  d.cycles = cycles;
  int rc = run_impl(ctx, cycles, d, (ctx->opt.flags & RTLSIM_F_DIGEST) != 0);
  if (rc) return rc;
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_sync(rtlsim_ctx *ctx) {
  if (!ctx) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->host_only) return RTLSIM_OK;
  CK(cudaStreamSynchronize(ctx->st));
  CK(cudaStreamSynchronize(ctx->st_h2d));
  CK(cudaStreamSynchronize(ctx->st_d2h));
  return RTLSIM_OK;
}

// ------------------------------------------------------------ registers --
extern "C" int rtlsim_get_regs(rtlsim_ctx *ctx, uint32_t *regs) {
  if (!ctx || !regs) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "get_regs before bind");
  return export_regs(ctx, regs);
}

extern "C" int rtlsim_set_regs(rtlsim_ctx *ctx, const uint32_t *regs) {
  if (!ctx || !regs) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "set_regs before bind");
  Program &G = ctx->prog;
  if (!G.RW) return RTLSIM_OK;
  CK(cudaSetDevice(ctx->device));
  uint32_t *tmp = nullptr;
  CK(cudaMallocAsync((void **)&tmp, (size_t)ctx->N * G.RW * 4, ctx->st));
  CK(cudaMemcpyAsync(tmp, regs, (size_t)ctx->N * G.RW * 4, cudaMemcpyHostToDevice, ctx->st));
  CK(launch_regs_import(tmp, G.RW, ctx->d_regmap, G.RW, (uint32_t)ctx->N, ctx->N_pad, ctx->state[ctx->cycle & 1],
                        ctx->st));
  ctx->launches++;
  CK(cudaFreeAsync(tmp, ctx->st));
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_reset(rtlsim_ctx *ctx) {
  if (!ctx) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "reset before bind");
  CK(cudaSetDevice(ctx->device));
  int rc = reset_regs(ctx);
  if (rc) return rc;
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_coverage(rtlsim_ctx *ctx, uint32_t *bitmap, int clear) {
  if (!ctx || !bitmap) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (!(ctx->opt.flags & RTLSIM_F_COVERAGE)) return arg_fail(ctx, RTLSIM_E_STATE, "loaded without RTLSIM_F_COVERAGE");
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "coverage before bind");
  Program &G = ctx->prog;
  if (!G.RW) return RTLSIM_OK;
  CK(cudaSetDevice(ctx->device));
  CK(cudaMemcpyAsync(bitmap, ctx->d_cov, (size_t)G.RW * 4, cudaMemcpyDeviceToHost, ctx->st));
  if (clear) CK(cudaMemsetAsync(ctx->d_cov, 0, (size_t)G.RW * 4, ctx->st));
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_get_mems(rtlsim_ctx *ctx, uint32_t *mems) {
  if (!ctx || !mems) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "get_mems before bind");
  Program &G = ctx->prog;
  if (!G.MR) return RTLSIM_OK;
  CK(cudaSetDevice(ctx->device));
  uint32_t *tmp = nullptr;
  CK(cudaMallocAsync((void **)&tmp, (size_t)ctx->N * G.MR * 4, ctx->st));
  CK(launch_mem_export(ctx->d_mem, G.MR, (uint32_t)ctx->N, ctx->N_pad, tmp, ctx->st));
  ctx->launches++;
  CK(cudaMemcpyAsync(mems, tmp, (size_t)ctx->N * G.MR * 4, cudaMemcpyDeviceToHost, ctx->st));
  CK(cudaFreeAsync(tmp, ctx->st));
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

extern "C" int rtlsim_reg_digest(rtlsim_ctx *ctx, uint64_t *digest) {
  if (!ctx || !digest) return RTLSIM_E_ARG;
  if (ctx->failed) return arg_fail(ctx, RTLSIM_E_STATE, ctx->err);
  if (ctx->src == SRC_NONE) return arg_fail(ctx, RTLSIM_E_STATE, "reg_digest before bind");
  Program &G = ctx->prog;
  CK(cudaSetDevice(ctx->device));
  unsigned long long *tmp = nullptr;
  CK(cudaMallocAsync((void **)&tmp, (size_t)ctx->N * 8, ctx->st));
  CK(launch_reg_digest(ctx->state[ctx->cycle & 1], ctx->d_regmap, G.RW, (uint32_t)ctx->N, ctx->N_pad, tmp, ctx->st));
  ctx->launches++;
  CK(cudaMemcpyAsync(digest, tmp, (size_t)ctx->N * 8, cudaMemcpyDeviceToHost, ctx->st));
  CK(cudaFreeAsync(tmp, ctx->st));
  CK(cudaStreamSynchronize(ctx->st));
  return RTLSIM_OK;
}

// ---------------------------------------------------------------- misc --
extern "C" int rtlsim_stats(const rtlsim_ctx *cctx, rtlsim_stats_t *st) {
  if (!cctx || !st) return RTLSIM_E_ARG;
  rtlsim_ctx *ctx = const_cast<rtlsim_ctx *>(cctx);
  if (!ctx->failed && !ctx->timed_pending.empty()) {
    int rc = fold_timing(ctx);
    if (rc) return rc;
  }
  const Program &G = ctx->prog;
  memset(st, 0, sizeof *st);
  st->n_ops = G.n_ops;
  st->n_signals = G.n_signals;
  st->n_regs = G.reg_q.size();
  st->word_ops = G.word_ops;
  st->n_desc = G.desc.size();
  st->n_steps = G.n_steps;
  st->n_partitions = G.n_partitions;
  st->b_floor = G.b_floor;
  st->b_state = G.b_state;
  st->b_part = G.b_part;
  st->b_spill = G.b_spill;
  st->n_live_ops = G.n_live_ops;
  st->live_word_ops = G.live_word_ops;
  st->rows_bit = G.rows[CLS_BIT]; st->rows_u8 = G.rows[CLS_U8];
  st->rows_u16 = G.rows[CLS_U16]; st->rows_u32 = G.rows[CLS_U32];
  st->xrows_bit = G.xrows[CLS_BIT]; st->xrows_u8 = G.xrows[CLS_U8];
  st->xrows_u16 = G.xrows[CLS_U16]; st->xrows_u32 = G.xrows[CLS_U32];
  st->smem_words = G.smem_words;
  st->op_lanes = G.L;
  st->chunk_cycles = ctx->Tc;
  st->tile_stimuli = 32;
  st->iw = G.IW; st->ow = G.OW; st->rw = G.RW;
  st->device_bytes = ctx->device_bytes;
  st->eval_ms = ctx->eval_ms;
  st->eval_launches = ctx->eval_launches;
  st->eval_stim_cycles = ctx->eval_stim_cycles;
  st->jit_compile_s = ctx->jit.compile_s;
  st->jit_cubin_bytes = ctx->jit.cubin_bytes;
  st->jit_sass_instructions = ctx->jit.sass_instructions;
  st->jit_tiles_per_cta = 0;
  st->tmem_cols = ctx->prog.tmem_cols;
  if (!ctx->jit.kern.empty() && ctx->N_pad)
    for (uint32_t q = 0; q < ctx->jit.kern.size(); q++)
      if (ctx->jit.kern[q]) st->jit_tiles_per_cta = std::max(st->jit_tiles_per_cta, jit_tiles_per_cta(ctx, ctx->jit, q));
  st->n_bitops = G.n_bitops; st->n_narrow = G.n_narrow; st->n_wide = G.n_wide;
  st->n_ld = G.n_ld; st->n_st = G.n_st;
  return RTLSIM_OK;
}

extern "C" uint64_t rtlsim_launch_count(const rtlsim_ctx *ctx) { return ctx ? ctx->launches : 0; }

extern "C" const char *rtlsim_last_error(const rtlsim_ctx *ctx) {
  return ctx ? ctx->err.c_str() : g_load_error.c_str();
}

extern "C" void rtlsim_free(rtlsim_ctx *ctx) {
  if (!ctx) return;
  if (!ctx->host_only) {
    cudaSetDevice(ctx->device);
    if (ctx->st) cudaStreamSynchronize(ctx->st);
    if (ctx->st_h2d) cudaStreamSynchronize(ctx->st_h2d);
    if (ctx->st_d2h) cudaStreamSynchronize(ctx->st_d2h);
    free_binding(ctx);
    jit_free(&ctx->jit);
    jit_free(&ctx->jit_dig);
    for (cudaStream_t x : ctx->dag_streams) cudaStreamDestroy(x);
    for (cudaEvent_t x : ctx->dag_events) cudaEventDestroy(x);
    if (ctx->dag_fork) cudaEventDestroy(ctx->dag_fork);
    for (auto &t : ctx->timed_pending) {
      cudaEventDestroy(t.a);
      cudaEventDestroy(t.b);
    }
    for (cudaEvent_t e : ctx->event_pool) cudaEventDestroy(e);
    for (void *p : ctx->dev_allocs) cudaFree(p);
    for (int b = 0; b < 2; b++) {
      if (ctx->ev_in_ready[b]) cudaEventDestroy(ctx->ev_in_ready[b]);
      if (ctx->ev_comp_done[b]) cudaEventDestroy(ctx->ev_comp_done[b]);
      if (ctx->ev_drain_done[b]) cudaEventDestroy(ctx->ev_drain_done[b]);
      if (ctx->ev_h2d_copied[b]) cudaEventDestroy(ctx->ev_h2d_copied[b]);
    }
    if (ctx->ev_start) cudaEventDestroy(ctx->ev_start);
    if (ctx->st_h2d) cudaStreamDestroy(ctx->st_h2d);
    if (ctx->st_d2h) cudaStreamDestroy(ctx->st_d2h);
    if (ctx->own_stream && ctx->st) cudaStreamDestroy(ctx->st);
    cudaGetLastError();
  }
  delete ctx;
}
