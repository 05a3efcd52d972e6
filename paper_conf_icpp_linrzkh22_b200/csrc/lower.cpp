// lower.cpp — lowering of the compiled descriptor schedule into the run-based
// micro-op stream of the v4 evaluator (program.h U_* classes).
//
// Same schedule, same slots, same semantics: every op of a step
// is still evaluated in that step; only its encoding changes so that the
// evaluator runs homogeneous loops without per-op decoding:
//   * narrow ops whose operand layouts equal the result layout become
//     class-specialized micro-ops (AND/OR/XOR/ADD/SUB/MUL, immediates, unary
//     COPY/NOT/NEG/SLICE/SEXT, MUX on a 1-bit select, unsigned compares, the
//     {bit, bit} concat);
//   * wide ops (> 32 bits) on 32-bit word rows become one micro-op per result
//     word (bitwise / MUX / funnel-shift words for CONCAT and SLICE) or a
//     word loop (ADD / SUB / NEG carry chain, unsigned compares); a missing
//     operand word reads the zero row, so every word is one uniform op;
//   * register / cross-partition / input row loads and register / net row
//     stores are batched several rows per warp instruction;
//   * everything else keeps its generic descriptor (U_GEN).
// The paper's kernels are transpiled straight-line code per partition
// (P:L438-672); this is the B200 counterpart of its "incremental memory
// allocation + index mapping" output: a compact op stream whose encoding
// fixes layouts per run instead of per instruction.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <string>

#include "program.h"

namespace rtlsim {
namespace {

inline uint32_t maskw(uint32_t w) { return w >= 32 ? 0xFFFFFFFFu : ((1u << w) - 1u); }
// mask shift of word i of a width-wd value: mask = 0xFFFFFFFF >> ms
inline uint32_t mshift(uint32_t wd, uint32_t i) {
  const uint32_t n = nwords(wd), rem = wd & 31u;
  return (i == n - 1 && rem) ? 32u - rem : 0u;
}
inline int e_idx(uint32_t lay) { return lay == LC_U8 ? 0 : lay == LC_U16 ? 1 : lay == LC_U32 ? 2 : -1; }

struct UOp {
  uint32_t cls;
  Desc q;
  double cost;
};

struct Lowerer {
  const Program &G;
  uint32_t zero_b;   // byte offset of the zero row
  std::vector<UOp> *out;

  void push(uint32_t cls, uint32_t x, uint32_t y, uint32_t z, uint32_t w, double cost) {
    out->push_back(UOp{cls, Desc{x, y, z, w}, cost});
  }
  std::map<std::string, uint64_t> *hist = nullptr;
  void gen(const Desc &q, double cost) {
    out->push_back(UOp{U_GEN, q, cost});
    if (!hist) return;
    const uint32_t code = q.x & 0xFFu;
    const char *ln[6] = {"U32", "BIT", "U16", "U8", "IMM", "BC"};
    char k[96];
    if (code < 32u) {
      snprintf(k, sizeof k, "N op%02u %s,%s,%s->%s", code, ln[(q.x >> 8) & 7u], ((q.w >> 11) & 1u) ? ln[(q.x >> 11) & 7u] : "-",
               ((q.w >> 12) & 1u) ? ln[(q.x >> 14) & 7u] : "-", ln[(q.x >> 17) & 7u]);
    } else if (code == CODE_WIDE) {
      const WideRec &r = G.wide[q.y];
      snprintf(k, sizeof k, "W op%02u %s,%s,%s wd%s", r.op, ln[r.lays & 0xFF], ln[(r.lays >> 8) & 0xFF], ln[(r.lays >> 16) & 0xFF],
               r.wd > 32 ? ">32" : "<=32");
    } else {
      snprintf(k, sizeof k, "M code%u", code);
    }
    (*hist)[k]++;
  }

  // byte address of word j of a U32-row operand (zero row beyond its words)
  uint32_t word(uint32_t off, uint32_t w, int64_t j) const {
    if (j < 0 || j >= (int64_t)nwords(w)) return zero_b;
    return 4u * (off + 32u * (uint32_t)j);
  }

  // any-layout narrow op (U_GX*): operand field = byte offset, or the value of an immediate
  bool gx(const Desc &q) {
    const uint32_t op = q.x & 0xFFu;
    const uint32_t la = (q.x >> 8) & 7u, lb = (q.x >> 11) & 7u, lc = (q.x >> 14) & 7u, ld = (q.x >> 17) & 7u;
    const uint32_t wd = (q.x >> 20) & 63u, wb = q.w & 63u, imm = (q.w >> 6) & 31u;
    const bool hb = (q.w >> 11) & 1u, hc = (q.w >> 12) & 1u;
    const uint32_t d = q.y & 0xFFFFu, a = q.y >> 16, b = q.z & 0xFFFFu, c = q.z >> 16;
    if (ld == LC_IMM || ld == LC_BCAST || la == LC_BCAST || (hb && lb == LC_BCAST) || (hc && lc == LC_BCAST)) return false;
    auto fld = [](uint32_t lay, uint32_t off) { return lay == LC_IMM ? off : 4u * off; };
    const uint32_t ms = (32u - wd) & 31u;
    const uint32_t x = 4u * d | la << 18 | (hb ? lb : LC_IMM) << 21 | (hc ? lc : LC_IMM) << 24 | ms << 27;
    const uint32_t fa = fld(la, a), fb = hb ? fld(lb, b) : 0u, fc = hc ? fld(lc, c) : 0u;
    int k = -1;
    switch (op) {
      case RTLSIM_OP_AND: k = 0; break;
      case RTLSIM_OP_OR: k = 1; break;
      case RTLSIM_OP_XOR: k = 2; break;
      case RTLSIM_OP_ADD: k = 3; break;
      case RTLSIM_OP_SUB: k = 4; break;
      default: break;
    }
    if (k >= 0 && hb && !hc) {
      push(U_GXLA + k, x, fa, fb, ld << 24, 22);
      return true;
    }
    if (op == RTLSIM_OP_COPY || op == RTLSIM_OP_NOT || op == RTLSIM_OP_SLICE) {
      push(U_GXUN + (op == RTLSIM_OP_COPY ? 0 : op == RTLSIM_OP_NOT ? 1 : 2), x, fa, 0,
           (op == RTLSIM_OP_SLICE ? imm : 0u) | ld << 24, 14);
      return true;
    }
    if (op == RTLSIM_OP_CONCAT && hb) {
      push(U_GXCAT, x, fa, fb, (wb & 31u) | ld << 24, 22);
      return true;
    }
    if (op == RTLSIM_OP_MUX && hb && hc) {
      push(U_GXMUX, x, fa, fb, fc | ld << 24, 28);
      return true;
    }
    if (op >= RTLSIM_OP_EQ && op <= RTLSIM_OP_GEU && hb) {
      push(U_GXCMP + (op - RTLSIM_OP_EQ), x, fa, fb, ld << 24, 22);
      return true;
    }
    return false;
  }

  bool narrow(const Desc &q) {
    const uint32_t op = q.x & 0xFFu;
    const uint32_t la = (q.x >> 8) & 7u, lb = (q.x >> 11) & 7u, lc = (q.x >> 14) & 7u, ld = (q.x >> 17) & 7u;
    const uint32_t wd = (q.x >> 20) & 63u, wa = q.x >> 26, imm = (q.w >> 6) & 31u;
    const bool hb = (q.w >> 11) & 1u, hc = (q.w >> 12) & 1u;
    uint32_t d = q.y & 0xFFFFu, a = q.y >> 16, b = q.z & 0xFFFFu, c = q.z >> 16;
    const int E = e_idx(ld);
    const uint32_t m = maskw(wd);
    int bi = -1;
    switch (op) {
      case RTLSIM_OP_AND: bi = 0; break;
      case RTLSIM_OP_OR: bi = 1; break;
      case RTLSIM_OP_XOR: bi = 2; break;
      case RTLSIM_OP_ADD: bi = 3; break;
      case RTLSIM_OP_SUB: bi = 4; break;
      default: break;   // MUL: generic-layout path (rare)
    }
    if (bi >= 0 && E >= 0 && hb && !hc) {
      uint32_t LA = la, LB = lb;
      if (LA == LC_IMM && LB == ld && bi != 4) {   // commutative: immediate second
        std::swap(a, b);
        std::swap(LA, LB);
      }
      if (LA == ld && LB == ld) {
        push(U_BIN + 3 * bi + E, 4 * d, 4 * a, 4 * b, m, 10);
        return true;
      }
      return false;
    }
    int uk = -1;
    uint32_t param = 0;
    switch (op) {
      case RTLSIM_OP_COPY: uk = 0; break;
      case RTLSIM_OP_NOT: uk = 1; break;
      case RTLSIM_OP_SLICE: uk = 3; param = imm; break;
      default: break;   // NEG, SEXT: generic-layout path (rare)
    }
    if (uk >= 0) {
      if (E >= 0 && la == ld) {
        push(U_UN + 3 * uk + E, 4 * d, 4 * a, param, m, 9);
        return true;
      }
      return false;
    }
    if (op == RTLSIM_OP_MUX) {
      if (E >= 0 && la == LC_BIT && lb == ld && lc == ld && hb && hc) {
        push(U_MUX + E, 4 * d | ((32u - wd) & 31u) << 24, 4 * a, 4 * b, 4 * c, 12);
        return true;
      }
      return false;
    }
    int ck = -1;
    switch (op) {
      case RTLSIM_OP_EQ: ck = 0; break;
      case RTLSIM_OP_NE: ck = 1; break;
      case RTLSIM_OP_LTU: ck = 2; break;
      case RTLSIM_OP_LEU: ck = 3; break;
      case RTLSIM_OP_GTU: ck = 4; break;
      case RTLSIM_OP_GEU: ck = 5; break;
      default: break;
    }
    if (ck >= 0) {
      const int EA = e_idx(la);
      if (ld == LC_BIT && EA >= 0 && lb == la && hb) {
        push(U_CMP + 3 * ck + EA, 4 * d, 4 * a, 4 * b, 0, 12);
        return true;
      }
      return false;
    }
    return false;
  }

  bool wide(const WideRec &r) {
    const uint32_t la = r.lays & 0xFFu, lb = (r.lays >> 8) & 0xFFu, lc = (r.lays >> 16) & 0xFFu;
    const uint32_t wd = r.wd, nd = nwords(wd);
    const uint32_t ld = wd == 1 ? LC_BIT : value_layout(wd, false);
    auto u32 = [](uint32_t l) { return l == LC_U32; };
    switch (r.op) {
      case RTLSIM_OP_AND: case RTLSIM_OP_OR: case RTLSIM_OP_XOR: {
        if (ld != LC_U32) return false;
        const int bi = r.op == RTLSIM_OP_AND ? 0 : r.op == RTLSIM_OP_OR ? 1 : 2;
        uint32_t A = r.a, B = r.b, LA = la, LB = lb, WA = r.wa, WB = r.wb;
        if (LA == LC_IMM) {
          std::swap(A, B);
          std::swap(LA, LB);
          std::swap(WA, WB);
        }
        if (!u32(LA)) return false;
        if (u32(LB)) {
          for (uint32_t i = 0; i < nd; i++)
            push(U_BIN + 3 * bi + 2, 4 * (r.d + 32 * i), word(A, WA, i), word(B, WB, i), 0xFFFFFFFFu >> mshift(wd, i), 10);
          return true;
        }
        return false;
      }
      case RTLSIM_OP_NOT: case RTLSIM_OP_COPY: {
        if (ld != LC_U32 || !u32(la)) return false;
        const int uk = r.op == RTLSIM_OP_COPY ? 0 : 1;
        for (uint32_t i = 0; i < nd; i++)
          push(U_UN + 3 * uk + 2, 4 * (r.d + 32 * i), word(r.a, r.wa, i), 0, 0xFFFFFFFFu >> mshift(wd, i), 9);
        return true;
      }
      case RTLSIM_OP_MUX: {
        if (ld != LC_U32 || la != LC_BIT || !u32(lb) || !u32(lc)) return false;
        for (uint32_t i = 0; i < nd; i++)
          push(U_MUX + 2, 4 * (r.d + 32 * i) | mshift(wd, i) << 24, 4 * r.a, word(r.b, r.wb, i), word(r.c, r.wc, i), 12);
        return true;
      }
      case RTLSIM_OP_CONCAT: {
        if (ld != LC_U32 || !u32(la) || !u32(lb)) return false;
        const uint32_t ws = r.wb >> 5, bs = r.wb & 31u;
        for (uint32_t i = 0; i < nd; i++) {
          const int64_t j = (int64_t)i - ws;
          uint32_t lo, hi, sh;
          if (bs == 0) {
            lo = word(r.a, r.wa, j);
            hi = zero_b;
            sh = 0;
          } else {
            lo = word(r.a, r.wa, j - 1);
            hi = word(r.a, r.wa, j);
            sh = 32 - bs;
          }
          push(U_FUN, 4 * (r.d + 32 * i) | mshift(wd, i) << 24, lo, hi, word(r.b, r.wb, i) | sh << 24, 13);
        }
        return true;
      }
      case RTLSIM_OP_SLICE: {
        if (ld != LC_U32 || !u32(la)) return false;
        const uint32_t ws = r.imm >> 5, bs = r.imm & 31u;
        for (uint32_t i = 0; i < nd; i++)
          push(U_FUN, 4 * (r.d + 32 * i) | mshift(wd, i) << 24, word(r.a, r.wa, i + ws), word(r.a, r.wa, i + ws + 1),
               zero_b | bs << 24, 13);
        return true;
      }
      case RTLSIM_OP_ADD: case RTLSIM_OP_SUB: case RTLSIM_OP_NEG: {
        if (ld != LC_U32 || !u32(la)) return false;
        uint32_t A = r.a, WA = r.wa, B = 0, WB = 0, sub = r.op != RTLSIM_OP_ADD;
        if (r.op == RTLSIM_OP_NEG) {   // 0 - a
          B = r.a;
          WB = r.wa;
          A = 0;
          WA = 0;
        } else {
          if (!u32(lb)) return false;
          B = r.b;
          WB = r.wb;
        }
        const uint32_t na = WA ? nwords(WA) : 0, nb = nwords(WB);
        push(U_WADD, 4 * r.d, WA ? 4 * A : zero_b, 4 * B, nd | std::min(na, 63u) << 6 | nb << 12 | sub << 18 | mshift(wd, nd - 1) << 24,
             8 + 9.0 * nd);
        return true;
      }
      case RTLSIM_OP_EQ: case RTLSIM_OP_NE: case RTLSIM_OP_LTU: case RTLSIM_OP_LEU: case RTLSIM_OP_GTU:
      case RTLSIM_OP_GEU: {
        if (ld != LC_BIT || !u32(la) || !u32(lb)) return false;
        const uint32_t na = nwords(r.wa), nb = nwords(r.wb), n = std::max(na, nb);
        push(U_WCMP, 4 * r.d, 4 * r.a, 4 * r.b, n | na << 6 | nb << 12 | (r.op - RTLSIM_OP_EQ) << 18, 8 + 8.0 * n);
        return true;
      }
      default:
        return false;
    }
  }

  void one(const Desc &q) {
    const uint32_t code = q.x & 0xFFu;
    if (code < 32u) {
      if (!narrow(q) && !gx(q)) {
        if (hist) gen(q, 0), out->pop_back();   // histogram only
        push(U_MIX + code, q.x, q.y, q.z, q.w, (code == RTLSIM_OP_DIVU || code == RTLSIM_OP_MODU) ? 80 : 50);
      }
      return;
    }
    if (code == CODE_LD_CONST) {   // constants are known here: immediate word stores
      const uint32_t nw = (q.x >> 12) & 63u;
      const bool bc = (q.x >> 18) & 1u;
      for (uint32_t i = 0; i < nw; i++) {
        const uint32_t v = G.const_pool[q.z + i];
        if (bc) push(U_CONSTB, 4 * (q.y + i), v, 0, 0, 4);
        else push(U_CONST, 4 * (q.y + 32 * i), v, 0, 0, 5);
      }
      return;
    }
    if (code == CODE_WIDE) {
      const WideRec &r = G.wide[q.y];
      if (!wide(r)) gen(q, 60 + 25.0 * nwords(std::max<uint32_t>(r.wd, std::max<uint32_t>(r.wa, r.wb))));
      return;
    }
    const uint32_t cls = (q.x >> 8) & 3u, nw = (q.x >> 12) & 63u;
    static const double row_cost[4] = {0.4, 0.8, 1.5, 3.0};
    int arena = -1;
    if (code == CODE_LD_REG) arena = 0;
    if (code == CODE_LD_X) arena = 1;
    if (code == CODE_LD_IN) arena = 2;
    if (arena >= 0) {
      const uint32_t n = cls == CLS_U32 ? nw : 1u;
      for (uint32_t i = 0; i < n; i++) push(U_LD + 4 * arena + cls, 4 * (q.y + 32 * i), q.z + i, 0, 0, row_cost[cls]);
      return;
    }
    if (code == CODE_ST_REG || code == CODE_ST_X) {
      const uint32_t lay = (q.x >> 18) & 7u;
      static const uint32_t lay_of[4] = {LC_BIT, LC_U8, LC_U16, LC_U32};
      if (lay == lay_of[cls]) {
        const uint32_t n = cls == CLS_U32 ? nw : 1u;
        const uint32_t ar = code == CODE_ST_REG ? 0u : 1u;
        for (uint32_t i = 0; i < n; i++)
          push(U_ST + 4 * ar + cls, 4 * (q.y + 32 * i), q.z + i, q.w + i, 0, row_cost[cls]);
        return;
      }
    }
    gen(q, 15 + 5.0 * nw);
  }
};

// execution order inside an op-lane: row loads (asynchronous) first, then
// compute grouped by class, stores last, generic descriptors at the end
inline uint32_t rank(uint32_t cls) {
  if (cls >= U_LD && cls < U_ST) return cls - U_LD;
  if (cls >= U_ST) return 200 + cls;
  if (cls == U_GEN) return 400;
  return 100 + cls;
}

}  // namespace

bool unrolled(uint32_t cls) {
  return ((cls >= U_BIN && cls < U_WADD) && cls != U_CONST) || (cls >= U_GXLA && cls < U_NCLASS);
}

// run header of a micro-op class (program.h G_* groups)
static Desc run_header(uint32_t cls, uint32_t n) {
  if (cls >= U_BIN && cls < U_BIN + 18) {
    const uint32_t bi = (cls - U_BIN) / 3, e = (cls - U_BIN) % 3;
    if (bi <= 2) {   // AND, OR, XOR
      static const uint32_t A[3] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0u}, B[3] = {0u, 0xFFFFFFFFu, 0xFFFFFFFFu};
      return Desc{G_LOG + e, n, A[bi], B[bi]};
    }
    return Desc{G_ARI + e, n, bi == 4 ? 0xFFFFFFFFu : 0u, bi == 4 ? 1u : 0u};   // ADD, SUB
  }
  if (cls >= U_UN && cls < U_UN + 15) {
    const uint32_t k = (cls - U_UN) / 3, e = (cls - U_UN) % 3;
    return Desc{G_UN + e, n, k == 1 ? 0xFFFFFFFFu : 0u, 0};   // COPY, NOT, SLICE (z = shift)
  }
  if (cls >= U_MUX && cls < U_MUX + 3) return Desc{G_MUX + (cls - U_MUX), n, 0, 0};
  if (cls >= U_CMP && cls < U_CMP + 18) return Desc{G_CMP + (cls - U_CMP) % 3, n, (cls - U_CMP) / 3, 0};
  if (cls == U_FUN) return Desc{G_FUN, n, 0, 0};
  if (cls == U_CONST) return Desc{G_CONST, n, 0, 0};
  if (cls == U_CONSTB) return Desc{G_CONSTB, n, 0, 0};
  if (cls == U_WADD) return Desc{G_WADD, n, 0, 0};
  if (cls == U_WCMP) return Desc{G_WCMP, n, 0, 0};
  if (cls >= U_LD && cls < U_ST) return Desc{G_LD, n, (cls - U_LD) % 4, (cls - U_LD) / 4};
  if (cls >= U_ST && cls < U_ST + 8) return Desc{G_ST, n, (cls - U_ST) % 4, (cls - U_ST) / 4};
  if (cls >= U_MIX && cls < U_MIX + 31) return Desc{G_MIX, n, cls - U_MIX, 0};
  if (cls >= U_GXLA && cls < U_GXLA + 5) return Desc{G_GXLA, n, cls - U_GXLA, 0};
  if (cls >= U_GXUN && cls < U_GXUN + 3) return Desc{G_GXUN, n, cls == U_GXUN + 1 ? 0xFFFFFFFFu : 0u, 0};
  if (cls == U_GXCAT) return Desc{G_GXCAT, n, 0, 0};
  if (cls == U_GXMUX) return Desc{G_GXMUX, n, 0, 0};
  if (cls >= U_GXCMP && cls < U_GXCMP + 6) return Desc{G_GXCMP, n, cls - U_GXCMP, 0};
  return Desc{G_GEN, n, 0, 0};
}

void lower_program(Program &G) {
  // zero row (32 words, 16-byte aligned) after the slots
  G.zero_off = (G.smem_words + 3u) & ~3u;
  G.smem_words = G.zero_off + 32u;
  const uint32_t L = G.L;
  G.ustream.clear();
  G.uptr.assign((size_t)G.n_steps * L + 1, 0);
  std::memset(G.u_class_count, 0, sizeof G.u_class_count);
  std::vector<UOp> ops;
  Lowerer lw{G, 4u * G.zero_off, &ops};
  std::map<std::string, uint64_t> hist;
  if (getenv("RTLSIM_HIST")) lw.hist = &hist;
  for (uint32_t s = 0; s < G.n_steps; s++) {
    ops.clear();
    for (uint32_t k = G.step_ptr[(size_t)s * L]; k < G.step_ptr[(size_t)(s + 1) * L]; k++) lw.one(G.desc[k]);
    std::stable_sort(ops.begin(), ops.end(), [](const UOp &x, const UOp &y) { return rank(x.cls) < rank(y.cls); });
    double total = 0;
    for (const UOp &u : ops) total += u.cost;
    // contiguous, cost-balanced segments: each lane sees few classes
    size_t k = 0;
    double acc = 0;
    for (uint32_t l = 0; l < L; l++) {
      G.uptr[(size_t)s * L + l] = (uint32_t)G.ustream.size();
      const double target = total * (l + 1) / L;
      uint32_t cur = 0xFFFFFFFFu;
      size_t hdr = 0;
      // unrolled classes execute groups of kUnroll micro-ops: pad the run by
      // repeating its last micro-op (re-evaluating an op is idempotent: no op
      // of a step reads a slot written in the same step)
      auto close_run = [&]() {
        if (cur == 0xFFFFFFFFu || !unrolled(cur)) return;
        while (G.ustream[hdr].y % kUnroll) {
          const Desc last = G.ustream.back();
          G.ustream.push_back(last);
          G.ustream[hdr].y++;
        }
      };
      while (k < ops.size() && (l == L - 1 || acc + 0.5 * ops[k].cost <= target)) {
        const UOp &u = ops[k++];
        acc += u.cost;
        if (u.cls != cur) {
          close_run();
          cur = u.cls;
          hdr = G.ustream.size();
          G.ustream.push_back(run_header(u.cls, 0));
        }
        G.ustream[hdr].y++;
        G.ustream.push_back(u.q);
        G.u_class_count[u.cls]++;
      }
      close_run();
    }
  }
  G.uptr[(size_t)G.n_steps * L] = (uint32_t)G.ustream.size();
  if (getenv("RTLSIM_HIST")) {   // debugging aid: micro-op class histogram
    uint32_t mx = 0;
    for (size_t i = 0; i + 1 < G.uptr.size(); i++) mx = std::max(mx, G.uptr[i + 1] - G.uptr[i]);
    fprintf(stderr, "ustream %zu entries, max block %u\n", G.ustream.size(), mx);
    for (uint32_t c = 0; c < U_NCLASS; c++)
      if (G.u_class_count[c]) fprintf(stderr, "  class %3u: %llu\n", c, (unsigned long long)G.u_class_count[c]);
    std::vector<std::pair<uint64_t, std::string>> v;
    for (auto &kv : hist) v.push_back({kv.second, kv.first});
    std::sort(v.rbegin(), v.rend());
    for (size_t i = 0; i < v.size() && i < 40; i++) fprintf(stderr, "  GEN %8llu %s\n", (unsigned long long)v[i].first, v[i].second.c_str());
  }
}

}  // namespace rtlsim
