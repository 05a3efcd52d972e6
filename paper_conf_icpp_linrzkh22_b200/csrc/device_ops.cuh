// device_ops.cuh — device helpers shared by the interpreter kernel (kernels.cu)
// and the JIT runtime module (jit_rt.cu): slot layouts, operand fetch/store,
// the generic any-width op path, cp.async, the digest mixer.
#pragma once
#include <cstdint>

#include "kernels.h"
#include "program.h"

namespace rtlsim {

// ------------------------------------------------------------- helpers --
__device__ __forceinline__ uint32_t nw_of(uint32_t w) { return (w + 31u) >> 5; }

// Slot layouts in shared memory (per 32-stimulus tile, program.h LC_*):
//   LC_BIT   one packed word, bit `lane` = stimulus lane (written by ballot)
//   LC_U8    32 byte lanes (8 words);  LC_U16  32 half-word lanes (16 words)
//   LC_U32   one 32-word row per 32-bit word: word i of lane l at off+32i+l
//   LC_IMM   constant <= 16 bits: `off` is the value itself
//   LC_BCAST constant > 32 bits: one broadcast copy of its words
// Values are canonical (bits >= width are zero).

// store word i of a width-wd result (masking the top word); a 1-bit result is
// packed with a warp ballot and written by lane 0 (all lanes must call)
__device__ __forceinline__ void putw_l(uint32_t *sm, uint32_t off, uint32_t wd, uint32_t i, uint32_t x,
                                       uint32_t lane) {
  if (wd == 1) {
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, x & 1u);
    if (lane == 0) sm[off] = m;
    return;
  }
  const uint32_t n = nw_of(wd), rem = wd & 31u;
  if (i == n - 1 && rem) x &= (1u << rem) - 1u;
  if (wd <= 8) reinterpret_cast<uint8_t *>(sm)[4u * off + lane] = (uint8_t)x;
  else if (wd <= 16) reinterpret_cast<uint16_t *>(sm)[2u * off + lane] = (uint16_t)x;
  else sm[off + 32u * i + lane] = x;
}

// 4-byte asynchronous global -> shared copy (LDGSTS); completion is awaited
// once per step, just before the step barrier
__device__ __forceinline__ void cp_async4(void *smem_dst, const void *gsrc) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// copy the tile's segment of a class row (or nw consecutive u32 rows) into
// slot d, in the slot layout of its width class
__device__ __forceinline__ void ld_class(uint32_t *sm, uint32_t d, uint32_t cls, uint32_t nw, const Arena &ar,
                                         size_t row, uint32_t N, uint32_t tile, uint32_t lane) {
  uint8_t *smb = reinterpret_cast<uint8_t *>(sm);
  if (cls == CLS_U32) {
    #pragma unroll 1
    for (uint32_t i = 0; i < nw; i++) cp_async4(sm + d + 32u * i + lane, ar.u32 + (row + i) * N + tile * 32u + lane);
  } else if (cls == CLS_BIT) {
    if (lane == 0) cp_async4(sm + d, ar.bit + row * (N >> 5) + tile);
  } else if (cls == CLS_U8) {
    if (lane < 8) cp_async4(smb + 4u * d + 4u * lane, ar.u8 + row * N + tile * 32u + 4u * lane);
  } else {
    if (lane < 16)
      cp_async4(smb + 4u * d + 4u * lane, reinterpret_cast<const uint8_t *>(ar.u16 + row * N + tile * 32u) + 4u * lane);
  }
}

__device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
  z ^= z >> 30;
  z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27;
  z *= 0x94D049BB133111EBull;
  z ^= z >> 31;
  return z;
}

// Narrow fast path (every width <= 32): one 32-bit word per operand.
__device__ __forceinline__ uint32_t fetch1(const uint32_t *sm, uint32_t off, uint32_t lc, uint32_t lane) {
  switch (lc) {
    case LC_U32: return sm[off + lane];
    case LC_BIT: return (sm[off] >> lane) & 1u;
    case LC_U16: return reinterpret_cast<const uint16_t *>(sm)[2u * off + lane];
    case LC_U8: return reinterpret_cast<const uint8_t *>(sm)[4u * off + lane];
    default: return off;   // LC_IMM
  }
}

__device__ __forceinline__ void store1(uint32_t *sm, uint32_t d, uint32_t lc, uint32_t r, uint32_t lane) {
  switch (lc) {
    case LC_U32: sm[d + lane] = r; break;
    case LC_BIT: {
      const uint32_t m = __ballot_sync(0xFFFFFFFFu, r & 1u);
      if (lane == 0) sm[d] = m;
      break;
    }
    case LC_U16: reinterpret_cast<uint16_t *>(sm)[2u * d + lane] = (uint16_t)r; break;
    default: reinterpret_cast<uint8_t *>(sm)[4u * d + lane] = (uint8_t)r; break;
  }
}

// --------------------------------------------------------------- N1 --
// Generic path: any widths (1..1024), word loops over 32-bit words. Kept out
// of line so the hot loop below stays small in the instruction cache.
// word i of a wide-path operand: operands of <= 32 bits were fetched once
// into v (any layout); wider ones are U32 rows or broadcast constants
__device__ __forceinline__ uint32_t gw(const uint32_t *sm, uint32_t off, uint32_t w, uint32_t lay, uint32_t v,
                                       uint32_t i, bool sx, uint32_t lane) {
  const uint32_t n = nw_of(w), rem = w & 31u, top = n - 1u;
  uint32_t x;
  if (w <= 32u) {
    x = v;
  } else {
    const uint32_t j = i < n ? i : top;
    x = lay == LC_BCAST ? sm[off + j] : sm[off + 32u * j + lane];
  }
  if (i < n) {
    if (sx && i == top && rem && ((x >> (rem - 1)) & 1u)) x |= ~((1u << rem) - 1u);
    return x;
  }
  return sx ? 0u - ((x >> ((w - 1) & 31u)) & 1u) : 0u;   // x is the top word here
}

__device__ __noinline__ static void exec_wide(uint32_t *sm, const WideRec *__restrict__ rec, uint32_t lane) {
  const uint4 q0 = __ldg(reinterpret_cast<const uint4 *>(rec));       // op, wd|wa, wb|wc, imm
  const uint4 q1 = __ldg(reinterpret_cast<const uint4 *>(rec) + 1);   // d a b c
  const uint32_t lays = __ldg(reinterpret_cast<const uint32_t *>(rec) + 8);
  const uint32_t op = q0.x, imm = q0.w;
  const uint32_t wd = q0.y & 0xFFFFu, wa = q0.y >> 16, wb = q0.z & 0xFFFFu, wc = q0.z >> 16;
  const uint32_t d = q1.x, a = q1.y, b = q1.z, cc = q1.w;
  const uint32_t la = lays & 0xFFu, lb = (lays >> 8) & 0xFFu, lc = (lays >> 16) & 0xFFu;
  const uint32_t va = wa && wa <= 32u ? fetch1(sm, a, la, lane) : 0u;
  const uint32_t vb = wb && wb <= 32u ? fetch1(sm, b, lb, lane) : 0u;
  const uint32_t vc = wc && wc <= 32u ? fetch1(sm, cc, lc, lane) : 0u;
  const uint32_t nd = nw_of(wd);
#define GA(i, sx, ln) gw(sm, a, wa, la, va, (i), (sx), (ln))
#define GB(i, sx, ln) gw(sm, b, wb, lb, vb, (i), (sx), (ln))
#define GS(i, sx, ln) gw(sm, src, wsrc, lsrc, vsrc, (i), (sx), (ln))
#define PUT(i, v, ln) putw_l(sm, d, wd, (i), (v), (ln))
  switch (op) {
          case RTLSIM_OP_COPY:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, GA(i, false, lane), lane);
            break;
          case RTLSIM_OP_SEXT:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, GA(i, true, lane), lane);
            break;
          case RTLSIM_OP_NOT:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, ~GA(i, false, lane), lane);
            break;
          case RTLSIM_OP_AND:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++)
              PUT(i, GA(i, false, lane) & GB(i, false, lane), lane);
            break;
          case RTLSIM_OP_OR:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++)
              PUT(i, GA(i, false, lane) | GB(i, false, lane), lane);
            break;
          case RTLSIM_OP_XOR:
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++)
              PUT(i, GA(i, false, lane) ^ GB(i, false, lane), lane);
            break;
          case RTLSIM_OP_ADD:
          case RTLSIM_OP_SUB: {
            unsigned long long carry = (op == RTLSIM_OP_SUB) ? 1ull : 0ull;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              uint32_t x = GA(i, false, lane), y = GB(i, false, lane);
              if (op == RTLSIM_OP_SUB) y = ~y;
              unsigned long long t = (unsigned long long)x + y + carry;
              carry = t >> 32;
              PUT(i, (uint32_t)t, lane);
            }
            break;
          }
          case RTLSIM_OP_NEG: {
            unsigned long long carry = 1ull;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              unsigned long long t = (unsigned long long)(uint32_t)~GA(i, false, lane) + carry;
              carry = t >> 32;
              PUT(i, (uint32_t)t, lane);
            }
            break;
          }
          case RTLSIM_OP_MUL:
          case RTLSIM_OP_DIVU:
          case RTLSIM_OP_MODU: {
            unsigned long long x = GA(0, false, lane) |
                                   ((unsigned long long)GA(1, false, lane) << 32);
            unsigned long long y = GB(0, false, lane) |
                                   ((unsigned long long)GB(1, false, lane) << 32);
            unsigned long long r = op == RTLSIM_OP_MUL ? x * y : (y == 0ull ? 0ull : (op == RTLSIM_OP_DIVU ? x / y : x % y));
            PUT(0, (uint32_t)r, lane);
            if (nd > 1) PUT(1, (uint32_t)(r >> 32), lane);
            break;
          }
          case RTLSIM_OP_EQ: case RTLSIM_OP_NE: case RTLSIM_OP_LTU: case RTLSIM_OP_LEU:
          case RTLSIM_OP_GTU: case RTLSIM_OP_GEU: case RTLSIM_OP_LTS: case RTLSIM_OP_LES:
          case RTLSIM_OP_GTS: case RTLSIM_OP_GES: {
            const bool sg = op >= RTLSIM_OP_LTS;
            const uint32_t n = nw_of(wa > wb ? wa : wb);
            int cmp = 0;
            #pragma unroll 1
            for (int i = (int)n - 1; i >= 0 && cmp == 0; i--) {
              uint32_t x = GA((uint32_t)i, sg, lane), y = GB((uint32_t)i, sg, lane);
              if (x != y) {
                if (sg && i == (int)n - 1) cmp = ((int32_t)x < (int32_t)y) ? -1 : 1;
                else cmp = x < y ? -1 : 1;
              }
            }
            uint32_t t;
            switch (op) {
              case RTLSIM_OP_EQ: t = cmp == 0; break;
              case RTLSIM_OP_NE: t = cmp != 0; break;
              case RTLSIM_OP_LTU: case RTLSIM_OP_LTS: t = cmp < 0; break;
              case RTLSIM_OP_LEU: case RTLSIM_OP_LES: t = cmp <= 0; break;
              case RTLSIM_OP_GTU: case RTLSIM_OP_GTS: t = cmp > 0; break;
              default: t = cmp >= 0; break;
            }
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, i == 0 ? t : 0u, lane);
            break;
          }
          case RTLSIM_OP_SHL: {
            uint32_t sa = GB(0, false, lane);
            #pragma unroll 1
            for (uint32_t i = 1; i < nw_of(wb); i++) if (GB(i, false, lane)) sa = 0xFFFFFFFFu;
            const uint32_t ws = sa >> 5, bs = sa & 31u;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              uint32_t x = 0;
              if (sa < wd && i >= ws) {
                x = GA(i - ws, false, lane) << bs;
                if (bs && i > ws) x |= GA(i - ws - 1, false, lane) >> (32u - bs);
              }
              PUT(i, x, lane);
            }
            break;
          }
          case RTLSIM_OP_SHRL:
          case RTLSIM_OP_SHRA: {
            const bool sx = op == RTLSIM_OP_SHRA;
            const uint32_t W = wd > wa ? wd : wa;
            uint32_t sa = GB(0, false, lane);
            #pragma unroll 1
            for (uint32_t i = 1; i < nw_of(wb); i++) if (GB(i, false, lane)) sa = 0xFFFFFFFFu;
            if (sa > W) sa = W;   // beyond the context width: 0 / sign fill
            const uint32_t ws = sa >> 5, bs = sa & 31u;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              uint32_t x = GA(i + ws, sx, lane) >> bs;
              if (bs) x |= GA(i + ws + 1, sx, lane) << (32u - bs);
              PUT(i, x, lane);
            }
            break;
          }
          case RTLSIM_OP_MUX: {
            uint32_t sel = 0;
            #pragma unroll 1
            for (uint32_t i = 0; i < nw_of(wa); i++) sel |= GA(i, false, lane);
            const uint32_t src = sel ? b : cc, wsrc = sel ? wb : wc, lsrc = sel ? lb : lc, vsrc = sel ? vb : vc;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, GS(i, false, lane), lane);
            break;
          }
          case RTLSIM_OP_CONCAT: {
            const uint32_t ws = wb >> 5, bs = wb & 31u;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              uint32_t x = GB(i, false, lane);
              if (i >= ws) {
                x |= GA(i - ws, false, lane) << bs;
                if (bs && i > ws) x |= GA(i - ws - 1, false, lane) >> (32u - bs);
              }
              PUT(i, x, lane);
            }
            break;
          }
          case RTLSIM_OP_SLICE: {
            const uint32_t ws = imm >> 5, bs = imm & 31u;
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) {
              uint32_t x = GA(i + ws, false, lane) >> bs;
              if (bs) x |= GA(i + ws + 1, false, lane) << (32u - bs);
              PUT(i, x, lane);
            }
            break;
          }
          case RTLSIM_OP_REDAND:
          case RTLSIM_OP_REDOR:
          case RTLSIM_OP_REDXOR: {
            const uint32_t n = nw_of(wa), rem = wa & 31u;
            uint32_t t = op == RTLSIM_OP_REDAND ? 1u : 0u;
            #pragma unroll 1
            for (uint32_t i = 0; i < n; i++) {
              uint32_t x = GA(i, false, lane);
              if (op == RTLSIM_OP_REDAND) t &= (x == ((i == n - 1 && rem) ? ((1u << rem) - 1u) : 0xFFFFFFFFu));
              else if (op == RTLSIM_OP_REDOR) t |= (x != 0u);
              else t ^= (__popc(x) & 1u);
            }
            #pragma unroll 1
            for (uint32_t i = 0; i < nd; i++) PUT(i, i == 0 ? t : 0u, lane);
            break;
          }
          default:
            break;
  }
#undef GA
#undef GB
#undef GS
#undef PUT
}


}  // namespace rtlsim
