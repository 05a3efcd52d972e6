/*
 * oracle.h — plain CPU reference simulator for the levelized RTL IR.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load liboracle.so. The
 * product path (paper_conf_icpp_linrzkh22_b200/) never links, imports or
 * executes anything under oracle/, and this tree includes no product header.
 *
 * What it computes — the plain definition of cycle-based two-state RTL
 * simulation with batch stimulus (§2; Listing 1,
 * P:L229-245; full-cycle evaluation; one independent stimulus per
 * GPU thread; truncation on assignment; integer only,
 * P:L1004-1007), with the readings listed in DESIGN.md §3:
 *
 *   for each stimulus s (independent):
 *     R := reg_init (or regs_in[s])
 *     for c in 0..T-1:
 *       V[inputs]  := stim[s][c][.] & mask(width)        (reading 15)
 *       V[regs]    := R ;  V[consts] := const words
 *       for op in ops (given order):  V[dst] := EVAL(op) mod 2^w_dst
 *       out[s][c]  := V[outputs]                        (pre-edge, reading 3)
 *       R          := { V[reg_d[r]] mod 2^w_q[r] }      (non-blocking, 16c)
 *       digest[s][c] := DIGEST(out[s][c], R)            (check mode)
 *     regs_out[s] := R
 *
 * Parity pins: see tests/test_oracle_*.py and DESIGN.md §4. Every function in
 * oracle.c is pinned by at least one closed form, textbook sequence, paper
 * worked example or brute-force table.
 *
 * The opcode numbering below is the IR interchange format (mirrored, not
 * shared, with include/rtlsim.h and rtlgen/ir.py; a CPU test checks they
 * agree).
 */
#ifndef RTL_ORACLE_H
#define RTL_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  ORC_COPY = 0, ORC_SEXT = 1, ORC_NOT = 2, ORC_AND = 3, ORC_OR = 4, ORC_XOR = 5,
  ORC_ADD = 6, ORC_SUB = 7, ORC_NEG = 8, ORC_MUL = 9, ORC_DIVU = 10, ORC_MODU = 11,
  ORC_EQ = 12, ORC_NE = 13, ORC_LTU = 14, ORC_LEU = 15, ORC_GTU = 16, ORC_GEU = 17,
  ORC_LTS = 18, ORC_LES = 19, ORC_GTS = 20, ORC_GES = 21,
  ORC_SHL = 22, ORC_SHRL = 23, ORC_SHRA = 24, ORC_MUX = 25, ORC_CONCAT = 26,
  ORC_SLICE = 27, ORC_REDAND = 28, ORC_REDOR = 29, ORC_REDXOR = 30,
  ORC_MEMRD = 31, /* dst := MEM[imm][V[a]] (0 when V[a] >= depth): ARRSEL read */
  ORC_N_OPCODES = 32
};
enum { ORC_INPUT = 0, ORC_REG = 1, ORC_COMB = 2, ORC_CONST = 3 };

typedef struct {
  uint16_t opcode, part;
  uint32_t dst, a, b, c, imm;
} oracle_op;

typedef struct oracle_design oracle_design;

/* Build a design from the IR arrays (copied). Returns NULL and writes a
 * message into err[0..errlen) on malformed input. */
oracle_design *oracle_design_new(uint32_t n_signals, const uint16_t *width, const uint8_t *kind,
                                 uint32_t n_ops, const oracle_op *ops,
                                 uint32_t n_regs, const uint32_t *reg_q, const uint32_t *reg_d,
                                 const uint32_t *reg_init,
                                 uint32_t n_consts, const uint32_t *const_sig,
                                 const uint32_t *const_words,
                                 uint32_t n_inputs, const uint32_t *input_sig,
                                 uint32_t n_outputs, const uint32_t *output_sig,
                                 char *err, int errlen);
void oracle_design_free(oracle_design *d);

/* Memories (§3.1.1, Fig 5: ARRSEL — an array variable indexed by a
 * run-time value, v1[v2[2]]; reading 12). Memory m has depth[m]
 * entries of width[m] bits (ceil(width/32) words each), initial contents
 * init[] (all memories, entry-major, the same for every stimulus). Reads are
 * the ORC_MEMRD op (combinational, see oracle_eval_op's caller). Write port
 * p = {mem, addr, data, en} (signals): at the clock edge, after outputs are
 * sampled and register next-states computed from the pre-edge values, every
 * port with V[en] != 0 and V[addr] < depth writes zext/trunc(V[data]) to
 * entry V[addr]; ports apply in index order (a later port wins). Reads in a
 * cycle see the memory as it was at the start of the cycle (non-blocking,
 * like registers). Returns 0, or -1 with err on bad arguments. */
int oracle_design_set_mems(oracle_design *d, uint32_t n_mems, const uint16_t *width, const uint32_t *depth,
                           const uint32_t *init, uint32_t n_wports, const uint32_t *wports /* [n][4] */,
                           char *err, int errlen);
/* Words of all memories of one stimulus (sum depth * ceil(width/32)). */
uint64_t oracle_mw(const oracle_design *d);
/* Like oracle_simulate, plus the final memory contents mem_out [N][MW] (may
 * be NULL). */
int oracle_simulate_mem(const oracle_design *d, uint64_t N, uint64_t T, const uint32_t *stim,
                        const uint32_t *regs_in, uint32_t *out, uint32_t *regs_out, uint64_t *digest,
                        uint32_t *mem_out, int n_threads, char *err, int errlen);
uint32_t oracle_iw(const oracle_design *d);
uint32_t oracle_ow(const oracle_design *d);
uint32_t oracle_rw(const oracle_design *d);

/* Simulate N stimuli x T cycles. stim: [N][T][IW]. regs_in: [N][RW] or NULL
 * (NULL = reg_init for every stimulus). Outputs (each may be NULL):
 * out [N][T][OW], regs_out [N][RW], digest [N][T]. n_threads <= 1 runs the
 * plain single-threaded loop; > 1 splits the stimulus loop into contiguous
 * blocks (stimuli are independent). Returns 0, or -1 with err. */
int oracle_simulate(const oracle_design *d, uint64_t N, uint64_t T, const uint32_t *stim,
                    const uint32_t *regs_in, uint32_t *out, uint32_t *regs_out,
                    uint64_t *digest, int n_threads, char *err, int errlen);

/* One op on explicit operands (tests: per-op pins). Operands are word
 * arrays of ceil(w/32) little-endian u32 words; result has ceil(wd/32). */
int oracle_eval_op(uint32_t opcode, uint32_t wd, uint32_t imm,
                   const uint32_t *a, uint32_t wa, const uint32_t *b, uint32_t wb,
                   const uint32_t *c, uint32_t wc, uint32_t *result);

/* splitmix64 finalizer used by DIGEST (check mode). */
uint64_t oracle_mix64(uint64_t z);

#ifdef __cplusplus
}
#endif
#endif
