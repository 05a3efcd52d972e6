/*
 * oracle.c — plain, slow, obviously-correct CPU simulator of the levelized RTL
 * IR. TEST INFRASTRUCTURE ONLY (see oracle.h for who may use it and for the
 * algorithm, which follows PAPER.md Listing 1, and §2.2,
 * every op is evaluated every cycle, in the given order).
 *
 * Values are arrays of little-endian u32 words (ceil(w/32) per signal). Every
 * operation is computed by first extending operands into a scratch "big"
 * value at a stated width, computing with word or bit loops, and then
 * truncating to the destination width ("truncation will be applied",
 * P:L648-651). No blocking, fusion or reordering: one stimulus at a time,
 * one cycle at a time, one op at a time.
 *
 * The semantics of each opcode are the readings of DESIGN.md §3 (IEEE 1364
 * two-state context-width rules as inherited through Verilator):
 * W = max(wd, wa, wb) (shifts: max(wd, wa)); operands zero-extended unless
 * the op is signed; shifts >= width give 0 / sign fill; DIVU/MODU by 0 give 0.
 */
#include "oracle.h"

#include <pthread.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define BIGW 68 /* 2176 bits: enough for CONCAT of two 1024-bit values */

typedef struct {
  uint32_t w[BIGW];
} big_t;

struct oracle_design {
  uint32_t n_signals, n_ops, n_regs, n_consts, n_inputs, n_outputs;
  uint16_t *width;
  uint8_t *kind;
  oracle_op *ops;
  uint32_t *reg_q, *reg_d, *reg_init; /* reg_init: RW words */
  uint32_t *const_sig, *const_words;
  uint32_t *input_sig, *output_sig;
  uint64_t *off; /* word offset of each signal in a value vector */
  uint64_t total_words;
  uint32_t iw, ow, rw;
  /* memories (oracle_design_set_mems) */
  uint32_t n_mems, n_wports;
  uint16_t *mem_width;
  uint32_t *mem_depth, *mem_init, *wports;
  uint64_t *mem_off; /* word offset of each memory in a memory vector */
  uint64_t mw;       /* words of all memories */
};

static unsigned nw(unsigned bits) { return (bits + 31u) / 32u; }
static unsigned umax(unsigned a, unsigned b) { return a > b ? a : b; }

static int getbit(const big_t *x, unsigned i) { return (int)((x->w[i / 32] >> (i % 32)) & 1u); }

/* zero every bit at position >= bits among the first `words` words (the
 * words above are already zero) */
static void mask_range(big_t *x, unsigned bits, unsigned words) {
  for (unsigned i = 0; i < words && i < BIGW; i++) {
    unsigned lo = 32 * i;
    if (lo >= bits)
      x->w[i] = 0;
    else if (bits - lo < 32)
      x->w[i] &= (1u << (bits - lo)) - 1u;
  }
}

/* x := src (w_src bits) extended to `bits` bits (zero- or sign-extension),
 * or truncated when bits < w_src. Only the first max(nw(w_src), nw(bits))
 * words of x are defined (written); every reader below stays inside the
 * words its own width defines, so no other word is ever cleared or read. */
static void ext(big_t *x, const uint32_t *src, unsigned w_src, unsigned bits, int sign) {
  const unsigned n = nw(w_src), nb = nw(bits) > n ? nw(bits) : n;
  for (unsigned i = 0; i < nb; i++) x->w[i] = i < n ? src[i] : 0u;
  mask_range(x, w_src, n);
  if (sign && bits > w_src && getbit(x, w_src - 1)) /* set bits w_src .. bits-1 */
    for (unsigned i = w_src / 32; i < nb; i++)
      x->w[i] |= (32 * i >= w_src) ? 0xFFFFFFFFu : ~((1u << (w_src % 32)) - 1u);
  mask_range(x, bits, nb);
}

/* r := x >> s on `words`-word values: bit i of r = bit i+s of x (0 above
 * the x's words). r and x are distinct. */
static void shr_words(big_t *r, const big_t *x, unsigned words, unsigned s) {
  const unsigned q = s / 32, k = s % 32;
  for (unsigned i = 0; i < words; i++) {
    uint32_t lo = i + q < words ? x->w[i + q] : 0u;
    uint32_t hi = i + q + 1 < words ? x->w[i + q + 1] : 0u;
    r->w[i] = k ? (lo >> k) | (hi << (32 - k)) : lo;
  }
}

/* r := x << s on `words`-word values: bit i of r = bit i-s of x (0 below
 * s). r and x are distinct. */
static void shl_words(big_t *r, const big_t *x, unsigned words, unsigned s) {
  const unsigned q = s / 32, k = s % 32;
  for (unsigned i = 0; i < words; i++) {
    uint32_t hi = i >= q ? x->w[i - q] : 0u;
    uint32_t lo = i >= q + 1 ? x->w[i - q - 1] : 0u;
    r->w[i] = k ? (hi << k) | (lo >> (32 - k)) : hi;
  }
}

/* x == 0 over its first `words` words */
static int is_zero(const big_t *x, unsigned words) {
  for (unsigned i = 0; i < words; i++)
    if (x->w[i]) return 0;
  return 1;
}

/* unsigned compare of two values (both extended to `words` words): -1, 0, 1 */
static int ucmp(const big_t *x, const big_t *y, unsigned words) {
  for (int i = (int)words - 1; i >= 0; i--) {
    if (x->w[i] != y->w[i]) return x->w[i] < y->w[i] ? -1 : 1;
  }
  return 0;
}

/* shift amount as an unsigned integer, saturated to 0xFFFFFFFF when it does
 * not fit in 32 bits (the shift operand is self-determined, reading 9) */
static uint32_t shamt(const uint32_t *b, unsigned wb) {
  big_t x;
  ext(&x, b, wb, wb, 0);
  for (unsigned i = 1; i < nw(wb); i++)
    if (x.w[i]) return 0xFFFFFFFFu;
  return x.w[0];
}

static uint64_t to_u64(const uint32_t *a, unsigned wa) {
  big_t x;
  ext(&x, a, wa, wa, 0);
  return (uint64_t)x.w[0] | (nw(wa) > 1 ? (uint64_t)x.w[1] << 32 : 0);
}

/* r's first two words := v (r is cleared by the caller) */
static void from_u64(big_t *r, uint64_t v) {
  r->w[0] = (uint32_t)v;
  r->w[1] = (uint32_t)(v >> 32);
}

static int is_signed_cmp(unsigned opc) {
  return opc == ORC_LTS || opc == ORC_LES || opc == ORC_GTS || opc == ORC_GES;
}

/* EVAL(op) mod 2^wd — DESIGN.md §3 table, one case per opcode. */
int oracle_eval_op(uint32_t opc, uint32_t wd, uint32_t imm, const uint32_t *a, uint32_t wa,
                   const uint32_t *b, uint32_t wb, const uint32_t *c, uint32_t wc,
                   uint32_t *result) {
  big_t x, y, r;
  unsigned W = umax(wd, umax(wa, b ? wb : 0));
  /* words of r any case below can write: every operand width, a CONCAT of
   * a and b, and two words for the 64-bit MUL/DIVU/MODU results */
  unsigned RN = nw(umax(umax(W, c ? wc : 0), umax(wa + (b ? wb : 0), 64)));
  if (RN > BIGW) RN = BIGW;
  for (unsigned i = 0; i < RN; i++) r.w[i] = 0;
  switch (opc) {
    case ORC_COPY: /* zext(a) mod 2^wd */
      ext(&r, a, wa, wd, 0);
      break;
    case ORC_SEXT: /* sext_{wa}(a) mod 2^wd */
      ext(&r, a, wa, umax(wa, wd), 1);
      break;
    case ORC_NOT: /* (~zext_W(a)) mod 2^wd: bits above wa become 1 */
      ext(&x, a, wa, W, 0);
      for (unsigned i = 0; i < nw(W); i++) r.w[i] = ~x.w[i];
      break;
    case ORC_AND:
    case ORC_OR:
    case ORC_XOR:
      ext(&x, a, wa, W, 0);
      ext(&y, b, wb, W, 0);
      for (unsigned i = 0; i < nw(W); i++)
        r.w[i] = opc == ORC_AND ? (x.w[i] & y.w[i])
                 : opc == ORC_OR ? (x.w[i] | y.w[i])
                                 : (x.w[i] ^ y.w[i]);
      break;
    case ORC_ADD:
    case ORC_SUB: { /* (a +- b) mod 2^wd; SUB = a + ~b + 1 */
      ext(&x, a, wa, W, 0);
      ext(&y, b, wb, W, 0);
      uint64_t carry = opc == ORC_SUB ? 1 : 0;
      for (unsigned i = 0; i < nw(W); i++) {
        uint64_t yy = opc == ORC_SUB ? (uint64_t)(uint32_t)~y.w[i] : (uint64_t)y.w[i];
        uint64_t s = (uint64_t)x.w[i] + yy + carry;
        r.w[i] = (uint32_t)s;
        carry = s >> 32;
      }
      break;
    }
    case ORC_NEG: { /* (0 - a) mod 2^wd = ~a + 1 */
      ext(&x, a, wa, W, 0);
      uint64_t carry = 1;
      for (unsigned i = 0; i < nw(W); i++) {
        uint64_t s = (uint64_t)(uint32_t)~x.w[i] + carry;
        r.w[i] = (uint32_t)s;
        carry = s >> 32;
      }
      break;
    }
    case ORC_MUL: /* (a*b) mod 2^wd, all widths <= 64 (reading 11) */
      if (wd > 64 || wa > 64 || wb > 64) return -1;
      from_u64(&r, to_u64(a, wa) * to_u64(b, wb));
      break;
    case ORC_DIVU:
    case ORC_MODU: { /* b == 0 -> 0 (reading 8) */
      if (wd > 64 || wa > 64 || wb > 64) return -1;
      uint64_t xa = to_u64(a, wa), yb = to_u64(b, wb);
      from_u64(&r, yb == 0 ? 0 : (opc == ORC_DIVU ? xa / yb : xa % yb));
      break;
    }
    case ORC_EQ: case ORC_NE: case ORC_LTU: case ORC_LEU: case ORC_GTU: case ORC_GEU:
    case ORC_LTS: case ORC_LES: case ORC_GTS: case ORC_GES: {
      /* operands extended to max(wa, wb): zero (unsigned) or sign (signed) */
      unsigned wc2 = umax(wa, wb);
      int sg = is_signed_cmp(opc);
      ext(&x, a, wa, wc2, sg);
      ext(&y, b, wb, wc2, sg);
      int cmp;
      if (sg && getbit(&x, wc2 - 1) != getbit(&y, wc2 - 1))
        cmp = getbit(&x, wc2 - 1) ? -1 : 1; /* negative < non-negative */
      else
        cmp = ucmp(&x, &y, nw(wc2)); /* same sign: two's complement order = unsigned order */
      int t = 0;
      switch (opc) {
        case ORC_EQ: t = cmp == 0; break;
        case ORC_NE: t = cmp != 0; break;
        case ORC_LTU: case ORC_LTS: t = cmp < 0; break;
        case ORC_LEU: case ORC_LES: t = cmp <= 0; break;
        case ORC_GTU: case ORC_GTS: t = cmp > 0; break;
        default: t = cmp >= 0; break;
      }
      r.w[0] = (uint32_t)t;
      break;
    }
    case ORC_SHL: { /* b >= wd -> 0; else (zext_W(a) << b) mod 2^wd */
      unsigned Ws = umax(wd, wa);
      uint32_t s = shamt(b, wb);
      ext(&x, a, wa, Ws, 0);
      if (s < wd) shl_words(&r, &x, nw(Ws), s);
      break;
    }
    case ORC_SHRL: { /* b >= W -> 0; else zext_W(a) >> b */
      unsigned Ws = umax(wd, wa);
      uint32_t s = shamt(b, wb);
      ext(&x, a, wa, Ws, 0);
      if (s < Ws) shr_words(&r, &x, nw(Ws), s);
      break;
    }
    case ORC_SHRA: { /* x = sext_{wa->W}(a); b >= W -> all sign; else x >>a b */
      /* bit i < W of the result is bit i+s of x, or the sign when i+s >= W:
       * sign-extend a further, to W + min(s, W) bits, and shift right */
      unsigned Ws = umax(wd, wa);
      uint32_t s = shamt(b, wb);
      if (s > Ws) s = Ws;
      ext(&x, a, wa, Ws + s, 1);
      shr_words(&r, &x, nw(Ws + s), s);
      break;
    }
    case ORC_MUX: /* a = select (any width), b = then, c = else */
      ext(&x, a, wa, wa, 0);
      if (!is_zero(&x, nw(wa)))
        ext(&r, b, wb, wd, 0);
      else
        ext(&r, c, wc, wd, 0);
      break;
    case ORC_CONCAT: /* ((a << wb) | b) mod 2^wd */
      ext(&x, a, wa, wa + wb, 0);
      ext(&y, b, wb, wb, 0);
      shl_words(&r, &x, nw(wa + wb), wb);
      for (unsigned i = 0; i < nw(wb); i++) r.w[i] |= y.w[i];
      break;
    case ORC_SLICE: /* (a >> imm) mod 2^wd; imm + wd <= wa is validated */
      if (imm + wd > wa) return -1;
      ext(&x, a, wa, wa, 0);
      shr_words(&r, &x, nw(wa), imm);
      break;
    case ORC_REDAND:
    case ORC_REDOR:
    case ORC_REDXOR: { /* all / any / parity of the wa bits of a */
      ext(&x, a, wa, wa, 0);
      uint32_t all = 1, any = 0, par = 0;
      for (unsigned i = 0; i < nw(wa); i++) {
        uint32_t full = (32 * i + 32 <= wa) ? 0xFFFFFFFFu : (1u << (wa % 32)) - 1u;
        all &= x.w[i] == full;
        any |= x.w[i] != 0;
        for (unsigned k = 0; k < 32; k++) par ^= (x.w[i] >> k) & 1u;
      }
      r.w[0] = opc == ORC_REDAND ? all : opc == ORC_REDOR ? any : par;
      break;
    }
    default:
      return -1;
  }
  mask_range(&r, wd, RN); /* truncation on assignment */
  for (unsigned i = 0; i < nw(wd); i++) result[i] = r.w[i];
  return 0;
}

/* splitmix64 finalizer (DIGEST) */
uint64_t oracle_mix64(uint64_t z) {
  z ^= z >> 30;
  z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27;
  z *= 0x94D049BB133111EBull;
  z ^= z >> 31;
  return z;
}

static void seterr(char *err, int errlen, const char *msg, long v) {
  if (err && errlen > 0) snprintf(err, (size_t)errlen, "%s (%ld)", msg, v);
}

static int op_arity(unsigned opc) {
  switch (opc) {
    case ORC_COPY: case ORC_SEXT: case ORC_NOT: case ORC_NEG: case ORC_SLICE:
    case ORC_REDAND: case ORC_REDOR: case ORC_REDXOR: case ORC_MEMRD:
      return 1;
    case ORC_MUX:
      return 3;
    default:
      return 2;
  }
}

void oracle_design_free(oracle_design *d) {
  if (!d) return;
  free(d->mem_width); free(d->mem_depth); free(d->mem_init); free(d->wports); free(d->mem_off);
  free(d->width); free(d->kind); free(d->ops); free(d->reg_q); free(d->reg_d);
  free(d->reg_init); free(d->const_sig); free(d->const_words); free(d->input_sig);
  free(d->output_sig); free(d->off); free(d);
}

#define DUP(dst, src, n, T)                                   \
  do {                                                        \
    (dst) = (T *)malloc(sizeof(T) * ((size_t)(n) + 1));       \
    if ((n) && (src)) memcpy((dst), (src), sizeof(T) * (size_t)(n)); \
  } while (0)

oracle_design *oracle_design_new(uint32_t n_signals, const uint16_t *width, const uint8_t *kind,
                                 uint32_t n_ops, const oracle_op *ops, uint32_t n_regs,
                                 const uint32_t *reg_q, const uint32_t *reg_d,
                                 const uint32_t *reg_init, uint32_t n_consts,
                                 const uint32_t *const_sig, const uint32_t *const_words,
                                 uint32_t n_inputs, const uint32_t *input_sig, uint32_t n_outputs,
                                 const uint32_t *output_sig, char *err, int errlen) {
  oracle_design *d = (oracle_design *)calloc(1, sizeof *d);
  d->n_signals = n_signals; d->n_ops = n_ops; d->n_regs = n_regs; d->n_consts = n_consts;
  d->n_inputs = n_inputs; d->n_outputs = n_outputs;
  DUP(d->width, width, n_signals, uint16_t);
  DUP(d->kind, kind, n_signals, uint8_t);
  DUP(d->ops, ops, n_ops, oracle_op);
  DUP(d->reg_q, reg_q, n_regs, uint32_t);
  DUP(d->reg_d, reg_d, n_regs, uint32_t);
  DUP(d->const_sig, const_sig, n_consts, uint32_t);
  DUP(d->input_sig, input_sig, n_inputs, uint32_t);
  DUP(d->output_sig, output_sig, n_outputs, uint32_t);
  d->off = (uint64_t *)malloc(sizeof(uint64_t) * ((size_t)n_signals + 1));
  uint64_t pos = 0;
  for (uint32_t s = 0; s < n_signals; s++) {
    if (width[s] < 1 || width[s] > 1024) { seterr(err, errlen, "width out of range at signal", s); goto fail; }
    d->off[s] = pos;
    pos += nw(width[s]);
  }
  d->off[n_signals] = pos;
  d->total_words = pos;
  uint32_t rw = 0, cw = 0;
  for (uint32_t r = 0; r < n_regs; r++) {
    if (reg_q[r] >= n_signals || reg_d[r] >= n_signals || kind[reg_q[r]] != ORC_REG) {
      seterr(err, errlen, "bad register", r); goto fail;
    }
    rw += nw(width[reg_q[r]]);
  }
  for (uint32_t k = 0; k < n_consts; k++) {
    if (const_sig[k] >= n_signals || kind[const_sig[k]] != ORC_CONST) { seterr(err, errlen, "bad const", k); goto fail; }
    cw += nw(width[const_sig[k]]);
  }
  d->rw = rw;
  DUP(d->reg_init, reg_init, rw, uint32_t);
  DUP(d->const_words, const_words, cw, uint32_t);
  d->iw = 0;
  for (uint32_t i = 0; i < n_inputs; i++) {
    if (input_sig[i] >= n_signals || kind[input_sig[i]] != ORC_INPUT) { seterr(err, errlen, "bad input", i); goto fail; }
    d->iw += nw(width[input_sig[i]]);
  }
  d->ow = 0;
  for (uint32_t o = 0; o < n_outputs; o++) {
    if (output_sig[o] >= n_signals) { seterr(err, errlen, "bad output", o); goto fail; }
    d->ow += nw(width[output_sig[o]]);
  }
  /* ops must come in topological order: each COMB operand defined by an
   * earlier op, each COMB signal defined exactly once (reading 13) */
  {
    uint8_t *def = (uint8_t *)calloc(n_signals + 1, 1);
    for (uint32_t i = 0; i < n_ops; i++) {
      const oracle_op *o = &ops[i];
      if (o->opcode >= ORC_N_OPCODES || o->dst >= n_signals || kind[o->dst] != ORC_COMB || def[o->dst]) {
        free(def); seterr(err, errlen, "bad op destination", i); goto fail;
      }
      uint32_t srcs[3] = {o->a, o->b, o->c};
      for (int k = 0; k < op_arity(o->opcode); k++) {
        uint32_t s = srcs[k];
        if (s >= n_signals || (kind[s] == ORC_COMB && !def[s])) {
          free(def); seterr(err, errlen, "operand not defined before use in op", i); goto fail;
        }
      }
      def[o->dst] = 1;
    }
    for (uint32_t s = 0; s < n_signals; s++)
      if (kind[s] == ORC_COMB && !def[s]) { free(def); seterr(err, errlen, "undriven comb signal", s); goto fail; }
    free(def);
  }
  return d;
fail:
  oracle_design_free(d);
  return NULL;
}

int oracle_design_set_mems(oracle_design *d, uint32_t n_mems, const uint16_t *width, const uint32_t *depth,
                           const uint32_t *init, uint32_t n_wports, const uint32_t *wports, char *err,
                           int errlen) {
  if (!d || (n_mems && (!width || !depth)) || (n_wports && !wports)) {
    seterr(err, errlen, "bad memory arguments", 0);
    return -1;
  }
  uint64_t mw = 0;
  for (uint32_t m = 0; m < n_mems; m++) {
    if (width[m] < 1 || width[m] > 1024 || depth[m] < 1) { seterr(err, errlen, "bad memory shape", m); return -1; }
    mw += (uint64_t)depth[m] * nw(width[m]);
  }
  for (uint32_t p = 0; p < n_wports; p++) {
    const uint32_t *w = wports + 4 * p;
    if (w[0] >= n_mems || w[1] >= d->n_signals || w[2] >= d->n_signals || w[3] >= d->n_signals) {
      seterr(err, errlen, "bad write port", p);
      return -1;
    }
  }
  for (uint32_t i = 0; i < d->n_ops; i++) {
    const oracle_op *o = &d->ops[i];
    if (o->opcode == ORC_MEMRD && (o->imm >= n_mems || d->width[o->dst] != width[o->imm])) {
      seterr(err, errlen, "MEMRD: no such memory or width differs", i);
      return -1;
    }
  }
  free(d->mem_width); free(d->mem_depth); free(d->mem_init); free(d->wports); free(d->mem_off);
  d->n_mems = n_mems;
  d->n_wports = n_wports;
  DUP(d->mem_width, width, n_mems, uint16_t);
  DUP(d->mem_depth, depth, n_mems, uint32_t);
  DUP(d->mem_init, init, mw, uint32_t);
  if (!init) memset(d->mem_init, 0, sizeof(uint32_t) * (size_t)mw);
  const size_t nwp = 4 * (size_t)n_wports;
  DUP(d->wports, wports, nwp, uint32_t);
  d->mem_off = (uint64_t *)malloc(sizeof(uint64_t) * ((size_t)n_mems + 1));
  uint64_t pos = 0;
  for (uint32_t m = 0; m < n_mems; m++) {
    d->mem_off[m] = pos;
    pos += (uint64_t)depth[m] * nw(width[m]);
  }
  d->mem_off[n_mems] = pos;
  d->mw = mw;
  return 0;
}

uint64_t oracle_mw(const oracle_design *d) { return d->mw; }

/* value of a (width wa) as an index: UINT32_MAX when it does not fit 32 bits */
static uint32_t as_index(const uint32_t *a, unsigned wa) { return shamt(a, wa); }

uint32_t oracle_iw(const oracle_design *d) { return d->iw; }
uint32_t oracle_ow(const oracle_design *d) { return d->ow; }
uint32_t oracle_rw(const oracle_design *d) { return d->rw; }

typedef struct {
  const oracle_design *d;
  uint64_t s0, s1, T;
  const uint32_t *stim, *regs_in;
  uint32_t *out, *regs_out;
  uint64_t *digest;
  uint32_t *mem_out;
  int rc;
} job_t;

/* Listing 1 for stimuli [s0, s1), one at a time. */
static void *run_block(void *arg) {
  job_t *j = (job_t *)arg;
  const oracle_design *d = j->d;
  uint32_t *V = (uint32_t *)calloc(d->total_words + 1, sizeof(uint32_t));
  uint32_t *R = (uint32_t *)calloc(d->rw + 1, sizeof(uint32_t));
  uint32_t *Rn = (uint32_t *)calloc(d->rw + 1, sizeof(uint32_t));
  uint32_t *M = (uint32_t *)calloc(d->mw + 1, sizeof(uint32_t));
  j->rc = 0;
  for (uint64_t s = j->s0; s < j->s1; s++) {
    /* R := reg_init, or the caller's per-stimulus state; M := memory init */
    memcpy(R, j->regs_in ? j->regs_in + s * d->rw : d->reg_init, sizeof(uint32_t) * d->rw);
    if (d->mw) memcpy(M, d->mem_init, sizeof(uint32_t) * d->mw);
    for (uint64_t c = 0; c < j->T; c++) {
      /* V[inputs] := stim[s][c] & mask(width) */
      const uint32_t *st = j->stim + (s * j->T + c) * d->iw;
      uint32_t k = 0;
      for (uint32_t i = 0; i < d->n_inputs; i++) {
        uint32_t sig = d->input_sig[i];
        big_t x;
        ext(&x, st + k, 32 * nw(d->width[sig]), d->width[sig], 0);
        for (unsigned t = 0; t < nw(d->width[sig]); t++) V[d->off[sig] + t] = x.w[t];
        k += nw(d->width[sig]);
      }
      /* V[regs] := R ; V[consts] := const words */
      k = 0;
      for (uint32_t r = 0; r < d->n_regs; r++) {
        uint32_t q = d->reg_q[r];
        for (unsigned t = 0; t < nw(d->width[q]); t++) V[d->off[q] + t] = R[k + t];
        k += nw(d->width[q]);
      }
      k = 0;
      for (uint32_t i = 0; i < d->n_consts; i++) {
        uint32_t sig = d->const_sig[i];
        big_t x;
        ext(&x, d->const_words + k, d->width[sig], d->width[sig], 0);
        for (unsigned t = 0; t < nw(d->width[sig]); t++) V[d->off[sig] + t] = x.w[t];
        k += nw(d->width[sig]);
      }
      /* evaluate every op, in the given (topological) order */
      for (uint32_t i = 0; i < d->n_ops; i++) {
        const oracle_op *o = &d->ops[i];
        int ar = op_arity(o->opcode);
        const uint32_t *pa = V + d->off[o->a];
        const uint32_t *pb = ar >= 2 ? V + d->off[o->b] : NULL;
        const uint32_t *pc = ar >= 3 ? V + d->off[o->c] : NULL;
        uint32_t wa = d->width[o->a];
        uint32_t wb = ar >= 2 ? d->width[o->b] : 0;
        uint32_t wc = ar >= 3 ? d->width[o->c] : 0;
        if (o->opcode == ORC_MEMRD) {
          /* ARRSEL read: entry V[a] of memory imm as it was at the start of
           * the cycle; an index >= depth reads 0 (reading 12) */
          if (o->imm >= d->n_mems) { j->rc = -1; goto done; }
          const uint32_t m = o->imm, n = nw(d->mem_width[m]), idx = as_index(pa, wa);
          for (unsigned t = 0; t < n; t++)
            V[d->off[o->dst] + t] = idx < d->mem_depth[m] ? M[d->mem_off[m] + (uint64_t)idx * n + t] : 0u;
          continue;
        }
        if (oracle_eval_op(o->opcode, d->width[o->dst], o->imm, pa, wa, pb, wb, pc, wc,
                           V + d->off[o->dst]) != 0) {
          j->rc = -1;
          goto done;
        }
      }
      /* out[s][c] := V[outputs] (pre-edge sampling, reading 3) */
      uint64_t dig = 0;
      k = 0;
      for (uint32_t o = 0; o < d->n_outputs; o++) {
        uint32_t sig = d->output_sig[o];
        for (unsigned t = 0; t < nw(d->width[sig]); t++) {
          uint32_t v = V[d->off[sig] + t];
          if (j->out) j->out[(s * j->T + c) * d->ow + k] = v;
          dig ^= oracle_mix64(((uint64_t)(k + 1) << 32) | v);
          k++;
        }
      }
      /* R_next := { V[reg_d[r]] mod 2^w_q }, all registers at once (16c) */
      k = 0;
      for (uint32_t r = 0; r < d->n_regs; r++) {
        uint32_t q = d->reg_q[r], dd = d->reg_d[r];
        big_t x;
        ext(&x, V + d->off[dd], d->width[dd], d->width[q], 0);
        for (unsigned t = 0; t < nw(d->width[q]); t++) {
          Rn[k] = x.w[t];
          dig ^= oracle_mix64(((uint64_t)(k + 1 + 0x80000000u) << 32) | Rn[k]);
          k++;
        }
      }
      if (j->digest) j->digest[s * j->T + c] = dig;
      /* memory write ports at the clock edge, in port order (a later port
       * wins); their signals are the pre-edge values of this cycle */
      for (uint32_t p = 0; p < d->n_wports; p++) {
        const uint32_t *w = d->wports + 4 * p;
        const uint32_t m = w[0], n = nw(d->mem_width[m]);
        big_t en, data;
        ext(&en, V + d->off[w[3]], d->width[w[3]], d->width[w[3]], 0);
        if (is_zero(&en, nw(d->width[w[3]]))) continue;
        const uint32_t idx = as_index(V + d->off[w[1]], d->width[w[1]]);
        if (idx >= d->mem_depth[m]) continue;
        ext(&data, V + d->off[w[2]], d->width[w[2]], d->mem_width[m], 0);
        for (unsigned t = 0; t < n; t++) M[d->mem_off[m] + (uint64_t)idx * n + t] = data.w[t];
      }
      memcpy(R, Rn, sizeof(uint32_t) * d->rw);
    }
    if (j->regs_out) memcpy(j->regs_out + s * d->rw, R, sizeof(uint32_t) * d->rw);
    if (j->mem_out && d->mw) memcpy(j->mem_out + s * d->mw, M, sizeof(uint32_t) * d->mw);
  }
done:
  free(V); free(R); free(Rn); free(M);
  return NULL;
}

int oracle_simulate(const oracle_design *d, uint64_t N, uint64_t T, const uint32_t *stim,
                    const uint32_t *regs_in, uint32_t *out, uint32_t *regs_out,
                    uint64_t *digest, int n_threads, char *err, int errlen) {
  return oracle_simulate_mem(d, N, T, stim, regs_in, out, regs_out, digest, NULL, n_threads, err, errlen);
}

int oracle_simulate_mem(const oracle_design *d, uint64_t N, uint64_t T, const uint32_t *stim,
                        const uint32_t *regs_in, uint32_t *out, uint32_t *regs_out, uint64_t *digest,
                        uint32_t *mem_out, int n_threads, char *err, int errlen) {
  if (!d || (N && T && d->iw && !stim)) { seterr(err, errlen, "bad arguments", 0); return -1; }
  if (n_threads < 1) n_threads = 1;
  if ((uint64_t)n_threads > N) n_threads = N ? (int)N : 1;
  job_t *jobs = (job_t *)calloc((size_t)n_threads, sizeof(job_t));
  pthread_t *th = (pthread_t *)calloc((size_t)n_threads, sizeof(pthread_t));
  for (int t = 0; t < n_threads; t++) {
    job_t *j = &jobs[t];
    j->d = d; j->T = T; j->stim = stim; j->regs_in = regs_in;
    j->out = out; j->regs_out = regs_out; j->digest = digest; j->mem_out = mem_out;
    j->s0 = N * (uint64_t)t / (uint64_t)n_threads;
    j->s1 = N * (uint64_t)(t + 1) / (uint64_t)n_threads;
  }
  int rc = 0;
  if (n_threads == 1) {
    run_block(&jobs[0]);
  } else {
    for (int t = 0; t < n_threads; t++) pthread_create(&th[t], NULL, run_block, &jobs[t]);
    for (int t = 0; t < n_threads; t++) pthread_join(th[t], NULL);
  }
  for (int t = 0; t < n_threads; t++)
    if (jobs[t].rc) rc = -1;
  if (rc) seterr(err, errlen, "unsupported operation (MUL/DIV > 64 bits, bad SLICE or MEMRD without memory)", 0);
  free(jobs); free(th);
  return rc;
}
