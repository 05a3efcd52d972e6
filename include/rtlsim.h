/*
 * rtlsim.h — C ABI of the B200-native batch-stimulus RTL simulator.
 *
 * The hot path of RTLflow (Lin et al., ICPP'22, PAPER.md): cycle-based
 * ("full-cycle") simulation of ONE levelized RTL design across a
 * batch of N independent stimuli, one GPU thread per stimulus,
 * every partition's combinational and sequential logic evaluated every clock
 * cycle (Listing 1). Outputs must equal the plain definition
 * (the CPU oracle, oracle/) bit for bit ("all signal outputs
 * match the golden reference").
 *
 * Conventions (all calls):
 *  - Every function returns RTLSIM_OK (0) or a negative rtlsim_status. No C++
 *    exception crosses the ABI. rtlsim_last_error() gives a message.
 *  - A value of width w is ceil(w/32) little-endian u32 words; bits >= w are
 *    zero in every output. IW / OW / RW = sum of ceil(w/32) over the inputs /
 *    outputs / registers, in IR order.
 *  - Argument and IR errors leave the ctx unchanged. A CUDA error makes the
 *    ctx sticky-failed: every later call except rtlsim_free returns
 *    RTLSIM_E_STATE. A ctx is not thread-safe; use one ctx per device.
 *  - Pointers documented "host" may be pageable or pinned (pinned buffers are
 *    copied with async DMA directly; pageable ones through pinned staging).
 *    Pointers documented "device" are CUDA device pointers on opt->device.
 */
#ifndef RTLSIM_H
#define RTLSIM_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  RTLSIM_OK = 0,
  RTLSIM_E_ARG = -1,         /* bad argument (NULL, size, range)                */
  RTLSIM_E_IR = -2,          /* malformed IR (driver count, kinds, widths, SLICE) */
  RTLSIM_E_COMB_LOOP = -3,   /* combinational cycle among ops (reading 13)      */
  RTLSIM_E_UNSUPPORTED = -4, /* MUL/DIVU/MODU wider than 64 bits (reading 11)   */
  RTLSIM_E_NOMEM = -5,       /* host or device allocation failed                */
  RTLSIM_E_CUDA = -6,        /* CUDA runtime error (ctx becomes sticky-failed)  */
  RTLSIM_E_STATE = -7,       /* wrong call order, or sticky failure             */
  RTLSIM_E_RANGE = -8        /* cycles beyond the bound stimulus (reading 14)   */
} rtlsim_status;

/* Signal kinds (§2: nodes of the RTL graph). */
enum { RTLSIM_INPUT = 0, RTLSIM_REG = 1, RTLSIM_COMB = 2, RTLSIM_CONST = 3 };

/* Opcodes (DESIGN.md §3 gives the exact two-state semantics; operands are
 * zero-extended to W = max(wd, wa, wb) unless stated, and every result is
 * truncated to the destination width). Numbering is the IR
 * interchange format (mirrored in rtlgen/ir.py). */
enum rtlsim_opcode {
  RTLSIM_OP_COPY = 0,   /* zext/trunc(a)                                     */
  RTLSIM_OP_SEXT = 1,   /* sext_{wa}(a)                                      */
  RTLSIM_OP_NOT = 2,    /* ~zext_W(a): high bits become 1 when wd > wa       */
  RTLSIM_OP_AND = 3, RTLSIM_OP_OR = 4, RTLSIM_OP_XOR = 5,
  RTLSIM_OP_ADD = 6, RTLSIM_OP_SUB = 7, RTLSIM_OP_NEG = 8,
  RTLSIM_OP_MUL = 9,    /* all widths <= 64                                  */
  RTLSIM_OP_DIVU = 10,  /* <= 64; b == 0 gives 0                             */
  RTLSIM_OP_MODU = 11,  /* <= 64; b == 0 gives 0                             */
  RTLSIM_OP_EQ = 12, RTLSIM_OP_NE = 13,                  /* 1-bit results   */
  RTLSIM_OP_LTU = 14, RTLSIM_OP_LEU = 15, RTLSIM_OP_GTU = 16, RTLSIM_OP_GEU = 17,
  RTLSIM_OP_LTS = 18, RTLSIM_OP_LES = 19, RTLSIM_OP_GTS = 20, RTLSIM_OP_GES = 21,
  RTLSIM_OP_SHL = 22,   /* b self-determined; b >= wd gives 0                */
  RTLSIM_OP_SHRL = 23,  /* b >= max(wd,wa) gives 0                           */
  RTLSIM_OP_SHRA = 24,  /* sext to max(wd,wa), b >= that width gives sign fill */
  RTLSIM_OP_MUX = 25,   /* a = select (any width, != 0), b = then, c = else  */
  RTLSIM_OP_CONCAT = 26,/* {a, b}: (a << wb) | b                             */
  RTLSIM_OP_SLICE = 27, /* a[imm + wd - 1 : imm]; imm + wd <= wa             */
  RTLSIM_OP_REDAND = 28, RTLSIM_OP_REDOR = 29, RTLSIM_OP_REDXOR = 30,
  RTLSIM_OP_MEMRD = 31  /* ARRSEL read: dst := MEM[imm][V[a]], 0 when V[a] >=
                           depth; wd = the memory's width (reading 12) */
};
#define RTLSIM_NONE 0xFFFFFFFFu
#define RTLSIM_MAX_WIDTH 1024

/* One op: V[dst] := EVAL(opcode, V[a], V[b], V[c], imm) mod 2^w_dst.
 * Unused operand fields are RTLSIM_NONE. `part` is the op's partition
 * (§3.2: macro tasks / partitions of the RTL graph). */
typedef struct {
  uint16_t opcode, part;
  uint32_t dst, a, b, c, imm;
} rtlsim_op;

/* The levelized design (borrowed only during rtlsim_load; copied). */
typedef struct {
  uint32_t n_signals;
  const uint16_t *width;       /* [n_signals], 1..1024                        */
  const uint8_t *kind;         /* [n_signals], RTLSIM_INPUT..RTLSIM_CONST     */
  uint32_t n_ops;
  const rtlsim_op *ops;        /* any order; must be acyclic, one driver per COMB */
  uint32_t n_regs;
  const uint32_t *reg_q;       /* [n_regs] REG signals                        */
  const uint32_t *reg_d;       /* [n_regs] any signal; q <= d mod 2^w_q       */
  const uint32_t *reg_init;    /* [RW] initial register words (all stimuli)   */
  uint32_t n_consts;
  const uint32_t *const_sig;   /* [n_consts] CONST signals                    */
  const uint32_t *const_words; /* [sum ceil(w/32)] constant words             */
  uint32_t n_inputs;
  const uint32_t *input_sig;   /* [n_inputs] INPUT signals: stimulus word order */
  uint32_t n_outputs;
  const uint32_t *output_sig;  /* [n_outputs] any signals: output word order  */
  uint32_t n_partitions;       /* ops[i].part < n_partitions; partition DAG acyclic */
  /* Memories (§3.1.1, Fig 5: ARRSEL, an array variable indexed at
   * run time, v1[v2[2]]; reading 12). All zero / NULL: none.
   * Memory m: mem_depth[m] entries of mem_width[m] bits, initial contents
   * mem_init (every memory's entries in order, ceil(w/32) words each; NULL =
   * all zero), the same for every stimulus. Reads: RTLSIM_OP_MEMRD ops (the
   * memory as it was at the start of the cycle). Write port p =
   * mem_wport[4p..4p+3] = {memory, address signal, data signal, enable
   * signal}: at the clock edge, with every register, if V[en] != 0 and
   * V[addr] < depth, entry V[addr] := V[data] zero-extended / truncated to the
   * memory width; ports apply in index order (a later port wins). Memory
   * state is per stimulus, laid out [entry word][N] in HBM. Supported with
   * RTLSIM_F_JIT (other backends: E_UNSUPPORTED); read and write addresses
   * at most 32 bits wide. */
  uint32_t n_mems;
  const uint16_t *mem_width;   /* [n_mems] 1..1024                             */
  const uint32_t *mem_depth;   /* [n_mems] >= 1                                */
  const uint32_t *mem_init;    /* [sum depth * ceil(w/32)] or NULL             */
  uint32_t n_wports;
  const uint32_t *mem_wport;   /* [n_wports * 4]                               */
} rtlsim_ir;

/* Option flags */
#define RTLSIM_F_DIGEST 0x1u      /* compute the per-(stimulus, cycle) digest   */
#define RTLSIM_F_NO_PIPELINE 0x2u /* host-buffer runs: serialise copy/compute   */
#define RTLSIM_F_GRAPH 0x4u       /* per-(cycle, partition) kernel nodes in a CUDA
                                     graph instead of one fused chunk kernel   */
#define RTLSIM_F_HOST_ONLY 0x8u   /* compile the schedule only; no device work
                                     (load/stats only; bind/run return E_STATE) */
#define RTLSIM_F_JIT 0x20u        /* specialized per-partition kernels: the
                                     schedule translated to PTX and compiled
                                     (nvPTXCompiler) at the first rtlsim_run*
                                     after a bind, specialised for the bound
                                     N rounded up to 32 (a rebind with another
                                     padded N recompiles; host-only contexts
                                     compile N-generic code at load); one
                                     launch per (cycle, partition),
                                     graph-captured                           */
#define RTLSIM_F_TIMING 0x10u     /* bracket every evaluator launch with CUDA
                                     events on the compute stream; totals in
                                     rtlsim_stats (eval_ms, eval_launches)     */
#define RTLSIM_F_STREAM 0x80u     /* ablation (Table 4): the per-(cycle,
                                     partition) launches of graph mode issued
                                     one by one into the stream, no graph     */
#define RTLSIM_F_V4 0x40u         /* reserved: the round-1 run-based micro-op
                                     evaluator, removed in round 2 (slower than
                                     the JIT and the descriptor interpreter on
                                     every config); rtlsim_load returns
                                     RTLSIM_E_UNSUPPORTED                     */
#define RTLSIM_F_COVERAGE 0x200u  /* toggle coverage (N5): after every cycle,
                                     bit j of register word k is set when it
                                     differs between R_c and R_{c+1} in any
                                     stimulus; read with rtlsim_coverage. The
                                     fused interpreter then runs per-(cycle,
                                     partition) launches (needs a cycle edge) */
#define RTLSIM_F_NO_DCE 0x100u    /* ablation: keep dead logic. By default ops
                                     whose value reaches no register D, no
                                     output and no live op are not evaluated
                                     (unobservable; Verilator's dead-code
                                     elimination)      */

typedef struct {
  int device;                /* CUDA device ordinal                           */
  void *cuda_stream;         /* cudaStream_t for compute, or NULL (own stream) */
  uint32_t op_lanes;         /* warps per CTA sharing one stimulus tile (0 = auto) */
  uint32_t chunk_cycles;     /* cycles per launch / pipeline chunk (0 = auto) */
  uint32_t flags;            /* RTLSIM_F_*                                    */
  uint32_t smem_limit;       /* bytes of shared memory per CTA (0 = device max);
                                long-lived values beyond it spill to HBM rows */
} rtlsim_options;

typedef struct {
  uint64_t n_ops, n_signals, n_regs;   /* design                              */
  uint64_t word_ops;         /* sum over ops of ceil(max(wd,wa,wb)/32)        */
  uint64_t n_desc;           /* descriptors incl. loads/stores per cycle      */
  uint64_t n_steps;          /* barrier-separated steps per cycle             */
  uint64_t n_partitions;
  double b_floor;            /* algorithmic HBM bytes per stimulus-cycle:
                                sum_regs 2 b(w) + sum_in b(w) + sum_out b(w)  */
  double b_state;            /* bytes the schedule moves per stimulus-cycle  */
  double b_part;             /* of which cross-partition nets                 */
  uint64_t rows_bit, rows_u8, rows_u16, rows_u32;    /* state arena rows      */
  uint64_t xrows_bit, xrows_u8, xrows_u16, xrows_u32;/* cross-partition rows  */
  uint64_t smem_words;       /* shared words per tile (per stimulus warp)     */
  uint32_t op_lanes, chunk_cycles, tile_stimuli, iw, ow, rw;
  uint64_t device_bytes;     /* device memory held by the ctx                 */
  double eval_ms;            /* RTLSIM_F_TIMING: summed evaluator launch time  */
  uint64_t eval_launches;    /* RTLSIM_F_TIMING: timed evaluator launches      */
  uint64_t eval_stim_cycles; /* RTLSIM_F_TIMING: stimulus-cycles they covered  */
  double jit_compile_s;      /* RTLSIM_F_JIT: PTX generation + compile seconds  */
  uint64_t jit_cubin_bytes;  /* RTLSIM_F_JIT: SASS bytes of all partition kernels */
  uint64_t n_bitops, n_narrow, n_wide, n_ld, n_st;   /* op stream composition    */
  double b_spill;            /* of b_state: spill stores + reloads of values that
                                exceed the smem budget (options.smem_limit) */
  uint64_t n_live_ops;       /* ops evaluated per cycle (n_ops minus dead logic) */
  uint64_t live_word_ops;    /* word_ops of the live ops                       */
  uint64_t jit_sass_instructions; /* RTLSIM_F_JIT: SASS instructions of all partition
                                kernels; straight-line code, so each is issued by
                                one warp per 32-stimulus tile per cycle:
                                / n_live_ops = warp-instructions per live op */
  uint32_t jit_tiles_per_cta;  /* RTLSIM_F_JIT: tiles per CTA of the largest launch
                                (warps of one op-lane that share each fetched
                                instruction)                                  */
  uint32_t tmem_cols;         /* (r2) TMEM columns per tile holding computed U32 values (RTLSIM_JIT_TMEM), else 0 */
} rtlsim_stats_t;

typedef struct rtlsim_ctx rtlsim_ctx;

/* Called by rtlsim_run_stream / bind_stream in cycle order.
 * producer: fill dst[N][nc][IW] (host, pinned) with stimulus cycles c0..c0+nc-1.
 * consumer: read out[N][nc][OW] (host) and digest[N][nc] (or NULL).
 * A non-zero return aborts the run with RTLSIM_E_ARG. The chunks already
 * simulated stay simulated: the cycle cursor and the register state are those
 * at the end of the last simulated chunk (for a consumer abort this can be one
 * chunk past the refused one, whose outputs were computed; rtlsim_stats does
 * not report the cursor — use rtlsim_reset / rtlsim_set_regs to restart from a
 * known state). The ctx stays usable (not sticky-failed).
 * PAPER.md §3.2.3 (Fig 11): stimulus groups flow through the
 * set_inputs (CPU) / evaluate (GPU) pipeline; these callbacks are its CPU
 * ends, producing inputs and consuming outputs one chunk (group) at a time. */
typedef int (*rtlsim_producer)(void *user, uint64_t c0, uint64_t nc, uint32_t *dst);
typedef int (*rtlsim_consumer)(void *user, uint64_t c0, uint64_t nc, const uint32_t *out,
                               const uint64_t *digest);

/* Validate, levelize and compile the design (the paper's
 * transpilation step, here a schedule + layout compiler), allocate device
 * state and upload descriptors. opt may be NULL (defaults). */
int rtlsim_load(const rtlsim_ir *ir, const rtlsim_options *opt, rtlsim_ctx **out);

/* Bind N stimuli x T cycles, host stimulus stim[N][T][IW] (borrowed until the
 * last run that reads it returns). Input bits above each input's width are
 * ignored (reading 15). Resets registers to reg_init and the cycle cursor to 0.
 * The stimulus is staged chunk by chunk (P:L919-963 pipeline), never copied
 * whole. N is 1..2097120 (65535 tiles of 32) per context: shard larger
 * batches over contexts / GPUs (§8(e)); a larger N returns RTLSIM_E_ARG. */
int rtlsim_bind(rtlsim_ctx *ctx, uint64_t N, uint64_t T, const uint32_t *stim);
/* Same with a DEVICE pointer to stim[N][T][IW] (resident in HBM; the
 * stimulus is already on the GPU, so the set_inputs stage of the P:L919-963
 * pipeline is a device-side transpose only). Borrowed until the last run that
 * reads it returns; E_ARG for N out of range. */
int rtlsim_bind_device(rtlsim_ctx *ctx, uint64_t N, uint64_t T, const uint32_t *stim_dev);
/* Same with a producer callback instead of a buffer: the CPU set_inputs task
 * of PAPER.md §3.2.3 (Fig 11) called per stimulus group (chunk of
 * cycles) into pinned staging, overlapped with the GPU's evaluation of the
 * previous chunk. prod must stay valid until the last run; a non-zero return
 * aborts that run (see rtlsim_producer). */
int rtlsim_bind_stream(rtlsim_ctx *ctx, uint64_t N, uint64_t T, rtlsim_producer prod, void *user);

/* Simulate `cycles` cycles c0..c0+cycles-1 from the ctx's cycle cursor c0
 * (E_RANGE if c0 + cycles > T; nothing is simulated). Host outputs (each may
 * be NULL): out[N][cycles][OW] (outputs sampled before the clock edge,
 * reading 3), regs[N][RW] after the last cycle, digest[N][cycles]. Blocking. */
int rtlsim_run(rtlsim_ctx *ctx, uint64_t cycles, uint32_t *out, uint32_t *regs, uint64_t *digest);
/* Same with DEVICE output buffers (either may be NULL): out_dev[N][cycles][OW],
 * digest_dev[N][cycles]. Asynchronous on the ctx's stream: call rtlsim_sync
 * before reading them. The per-cycle evaluation is the CUDA-graph schedule of
 * P:L852-917 (one node per partition per cycle). */
int rtlsim_run_device(rtlsim_ctx *ctx, uint64_t cycles, uint32_t *out_dev, uint64_t *digest_dev);
/* Same with a consumer callback receiving each chunk (host, transposed to
 * [N][nc][OW]; digest [N][nc] when loaded with RTLSIM_F_DIGEST): the output
 * drain end of the P:L919-963 pipeline. Blocking; a non-zero return aborts
 * the run (see rtlsim_consumer). */
int rtlsim_run_stream(rtlsim_ctx *ctx, uint64_t cycles, rtlsim_consumer cons, void *user);
/* Wait for everything queued on the ctx's streams (rtlsim_run_device). */
int rtlsim_sync(rtlsim_ctx *ctx);

/* Register state checkpoint: regs[N][RW] host (get/set), or reset to reg_init
 * (and memories to their initial contents) and cycle 0. The register state R
 * is what Listing 1's loop carries from cycle to cycle; E_STATE
 * before bind; set_regs does not move the cycle cursor. */
int rtlsim_get_regs(rtlsim_ctx *ctx, uint32_t *regs);
int rtlsim_set_regs(rtlsim_ctx *ctx, const uint32_t *regs);
int rtlsim_reset(rtlsim_ctx *ctx);

/* Toggle coverage bitmap (RTLSIM_F_COVERAGE contexts): bitmap[k] (host, RW
 * words) = OR over every simulated cycle c since the bind (or the last clear)
 * and every stimulus s of R_c[s][k] ^ R_{c+1}[s][k] — "bit toggled in any
 * stimulus". clear != 0 zeroes the device bitmap after reading. Multi-GPU:
 * the bitmaps of the stimulus shards combine by bitwise OR (north star: NCCL
 * gathers coverage; all_gather + OR, NCCL has no OR reduction). Errors:
 * E_STATE without the flag or before bind. */
int rtlsim_coverage(rtlsim_ctx *ctx, uint32_t *bitmap, int clear);
/* Memory contents mems[N][MW] (host; MW = sum over memories of depth x
 * ceil(width/32) words, memories and entries in IR order) after the last
 * simulated cycle: the ARRSEL array variables of PAPER.md §3.1.1 (Fig 5,
 * P:L496-531), per stimulus. E_STATE before bind. */
int rtlsim_get_mems(rtlsim_ctx *ctx, uint32_t *mems);
/* Per-stimulus digest of the current register state, digest[s] (host, N
 * words) = XOR_k mix(((k + 1 + 2^31) << 32) | R[s][k]) — the register half of
 * the per-cycle DIGEST, so N x 8 bytes identify every final
 * register state (the rank-0 gather of §8(e) collects these instead of the
 * registers themselves). P:L1128-1129: results compared per stimulus. */
int rtlsim_reg_digest(rtlsim_ctx *ctx, uint64_t *digest);

/* Compiled-design and run accounting (rtlsim_stats_t): op counts, the
 * algorithmic bytes per stimulus-cycle of SURVEY §8(d) (b_floor), the JIT's
 * SASS size and tiles per CTA, timing of evaluator launches (RTLSIM_F_TIMING).
 * Works on host-only contexts. E_ARG for NULL. */
int rtlsim_stats(const rtlsim_ctx *ctx, rtlsim_stats_t *st);
/* Kernel launches issued by this ctx since load (for the bench's gpu_launches). */
uint64_t rtlsim_launch_count(const rtlsim_ctx *ctx);
/* Message for the last failing call on ctx (NULL: the thread's last
 * rtlsim_load failure). Owned by the library; valid until the next call. */
const char *rtlsim_last_error(const rtlsim_ctx *ctx);
/* Release the ctx and everything it owns (device memory, streams, graphs,
 * JIT modules). NULL-safe; valid after a sticky failure. */
void rtlsim_free(rtlsim_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* RTLSIM_H */
