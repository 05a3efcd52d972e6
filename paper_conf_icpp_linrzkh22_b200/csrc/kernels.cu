// kernels.cu — hand-written sm_100a kernels of the simulator.
//
// N1 rtl_eval: the op-stream evaluator. One CTA = one tile of 32 stimuli
// (one thread per stimulus) x L op-lanes (warps that
// split the independent ops of each level, the paper's structure-level
// parallelism P:L159-162). Combinational values live in shared-memory slots,
// signal-major / stimulus-minor (slot word k of stimulus lane l at
// smem[k + l], the index mapping of P:L623-638 moved on-chip): every warp
// access is conflict-free. 1-bit values are packed, one u32 per 32 stimuli,
// written with __ballot_sync. Registers stream from width-class arenas in HBM
// (ping-pong buffers, non-blocking update). No tensor cores:
// nothing here is a dense contraction.
//
// N2/N3: stimulus / output transposes between the user layout [N][T][W]
// (stimulus-major) and the device layout [T][W][N] (coalesced per warp).
// N4: register init / import / export.
#include <algorithm>
#include <cstdint>

#include "device_ops.cuh"
#include "kernels.h"
#include "program.h"

namespace rtlsim {

__device__ __forceinline__ int32_t sx32(uint32_t x, uint32_t w) {
  const uint32_t sb = 1u << (w - 1u);
  return (int32_t)((x ^ sb) - sb);
}

// EVAL for narrow ops on canonical (zero-extended) operands; the caller
// truncates to wd. Semantics: DESIGN.md §3.
__device__ __forceinline__ uint32_t alu1(uint32_t op, uint32_t x, uint32_t y, uint32_t z, uint32_t wd, uint32_t wa,
                                         uint32_t wb, uint32_t imm) {
  switch (op) {
    case RTLSIM_OP_COPY: return x;
    case RTLSIM_OP_SEXT: return (uint32_t)sx32(x, wa);
    case RTLSIM_OP_NOT: return ~x;
    case RTLSIM_OP_AND: return x & y;
    case RTLSIM_OP_OR: return x | y;
    case RTLSIM_OP_XOR: return x ^ y;
    case RTLSIM_OP_ADD: return x + y;
    case RTLSIM_OP_SUB: return x - y;
    case RTLSIM_OP_NEG: return 0u - x;
    case RTLSIM_OP_MUL: return x * y;
    case RTLSIM_OP_DIVU: return y ? x / y : 0u;
    case RTLSIM_OP_MODU: return y ? x % y : 0u;
    case RTLSIM_OP_EQ: return x == y;
    case RTLSIM_OP_NE: return x != y;
    case RTLSIM_OP_LTU: return x < y;
    case RTLSIM_OP_LEU: return x <= y;
    case RTLSIM_OP_GTU: return x > y;
    case RTLSIM_OP_GEU: return x >= y;
    case RTLSIM_OP_LTS: return sx32(x, wa) < sx32(y, wb);
    case RTLSIM_OP_LES: return sx32(x, wa) <= sx32(y, wb);
    case RTLSIM_OP_GTS: return sx32(x, wa) > sx32(y, wb);
    case RTLSIM_OP_GES: return sx32(x, wa) >= sx32(y, wb);
    case RTLSIM_OP_SHL: return y >= wd ? 0u : x << y;
    case RTLSIM_OP_SHRL: return y >= 32u ? 0u : x >> y;
    case RTLSIM_OP_SHRA: return (uint32_t)(sx32(x, wa) >> (y > 31u ? 31u : y));
    case RTLSIM_OP_MUX: return x ? y : z;
    case RTLSIM_OP_CONCAT: return wb >= 32u ? y : ((x << wb) | y);
    case RTLSIM_OP_SLICE: return x >> imm;
    case RTLSIM_OP_REDAND: return x == (0xFFFFFFFFu >> (32u - wa));
    case RTLSIM_OP_REDOR: return x != 0u;
    default: return __popc(x) & 1u;   // REDXOR
  }
}

// ---- specialized narrow handlers (program.h HID_*): operand layouts are
// fixed per handler, so fetch / store compile to one shared-memory access
template <int X>
__device__ __forceinline__ uint32_t ldx(const uint32_t *sm, uint32_t off, uint32_t lane) {
  if constexpr (X == LC_U32) return sm[off + lane];
  else if constexpr (X == LC_U16) return reinterpret_cast<const uint16_t *>(sm)[2u * off + lane];
  else return reinterpret_cast<const uint8_t *>(sm)[4u * off + lane];
}
template <int X>
__device__ __forceinline__ void stx(uint32_t *sm, uint32_t off, uint32_t lane, uint32_t r) {
  if constexpr (X == LC_U32) sm[off + lane] = r;
  else if constexpr (X == LC_U16) reinterpret_cast<uint16_t *>(sm)[2u * off + lane] = (uint16_t)r;
  else reinterpret_cast<uint8_t *>(sm)[4u * off + lane] = (uint8_t)r;
}

__device__ __forceinline__ uint32_t bin_op(uint32_t op, uint32_t x, uint32_t y) {
  switch (op) {
    case RTLSIM_OP_AND: return x & y;
    case RTLSIM_OP_OR: return x | y;
    case RTLSIM_OP_XOR: return x ^ y;
    case RTLSIM_OP_ADD: return x + y;
    case RTLSIM_OP_SUB: return x - y;
    default: return x * y;   // MUL
  }
}

// kind: 0 binary X,X->X ; 1 binary X,IMM->X ; 2 unary X->X ; 3 MUX BIT,X,X->X ;
// 4 unsigned compare X,X->BIT
template <int X, int KIND>
__device__ __forceinline__ void fast_h(uint32_t *sm, const uint4 q, uint32_t op, uint32_t lane) {
  const uint32_t wd = (q.x >> 20) & 63u, m = 0xFFFFFFFFu >> (32u - wd);
  const uint32_t d = q.y & 0xFFFFu, a = q.y >> 16, b = q.z & 0xFFFFu, c = q.z >> 16;
  if constexpr (KIND == 0 || KIND == 1) {
    const uint32_t x = ldx<X>(sm, a, lane);
    const uint32_t y = KIND == 0 ? ldx<X>(sm, b, lane) : b;
    stx<X>(sm, d, lane, bin_op(op, x, y) & m);
  } else if constexpr (KIND == 2) {
    const uint32_t x = ldx<X>(sm, a, lane), wa = q.x >> 26;
    uint32_t r;
    switch (op) {
      case RTLSIM_OP_COPY: r = x; break;
      case RTLSIM_OP_NOT: r = ~x; break;
      case RTLSIM_OP_NEG: r = 0u - x; break;
      case RTLSIM_OP_SLICE: r = x >> ((q.w >> 6) & 31u); break;
      default: { const uint32_t sb = 1u << (wa - 1u); r = (x ^ sb) - sb; break; }   // SEXT
    }
    stx<X>(sm, d, lane, r & m);
  } else if constexpr (KIND == 3) {
    const uint32_t sel = (sm[a] >> lane) & 1u;
    stx<X>(sm, d, lane, ldx<X>(sm, sel ? b : c, lane));
  } else {
    const uint32_t x = ldx<X>(sm, a, lane), y = ldx<X>(sm, b, lane);
    bool t;
    switch (op) {
      case RTLSIM_OP_EQ: t = x == y; break;
      case RTLSIM_OP_NE: t = x != y; break;
      case RTLSIM_OP_LTU: t = x < y; break;
      case RTLSIM_OP_LEU: t = x <= y; break;
      case RTLSIM_OP_GTU: t = x > y; break;
      default: t = x >= y; break;   // GEU
    }
    const uint32_t bits = __ballot_sync(0xFFFFFFFFu, t);
    if (lane == 0) sm[d] = bits;
  }
}

__device__ __forceinline__ void fast_narrow(uint32_t *sm, const uint4 q, uint32_t hid, uint32_t op, uint32_t lane) {
  switch (hid) {
    case 1: fast_h<LC_U32, 0>(sm, q, op, lane); break;
    case 2: fast_h<LC_U16, 0>(sm, q, op, lane); break;
    case 3: fast_h<LC_U8, 0>(sm, q, op, lane); break;
    case 4: fast_h<LC_U32, 1>(sm, q, op, lane); break;
    case 5: fast_h<LC_U16, 1>(sm, q, op, lane); break;
    case 6: fast_h<LC_U8, 1>(sm, q, op, lane); break;
    case 7: fast_h<LC_U32, 2>(sm, q, op, lane); break;
    case 8: fast_h<LC_U16, 2>(sm, q, op, lane); break;
    case 9: fast_h<LC_U8, 2>(sm, q, op, lane); break;
    case 10: fast_h<LC_U32, 3>(sm, q, op, lane); break;
    case 11: fast_h<LC_U16, 3>(sm, q, op, lane); break;
    case 12: fast_h<LC_U8, 3>(sm, q, op, lane); break;
    case 13: fast_h<LC_U32, 4>(sm, q, op, lane); break;
    case 14: fast_h<LC_U16, 4>(sm, q, op, lane); break;
    default: fast_h<LC_U8, 4>(sm, q, op, lane); break;
  }
}

// bit-sliced op: 3-input truth table applied to packed words (32 stimuli)
__device__ __forceinline__ void exec_bit(uint32_t *sm, const uint4 q) {
  const uint32_t lut = q.x & 0xFFu, immf = q.x >> 8;
  const uint32_t fa = q.y >> 16, fb = q.z & 0xFFFFu, fc = q.z >> 16;
  const uint32_t x = (immf & 1u) ? 0u - (fa & 1u) : sm[fa];
  const uint32_t y = (immf & 2u) ? 0u - (fb & 1u) : sm[fb];
  const uint32_t z = (immf & 4u) ? 0u - (fc & 1u) : sm[fc];
  uint32_t r = 0;
#pragma unroll
  for (int k = 0; k < 8; k++) {
    const uint32_t t = ((k & 1) ? x : ~x) & ((k & 2) ? y : ~y) & ((k & 4) ? z : ~z);
    r |= t & (0u - ((lut >> k) & 1u));
  }
  sm[q.y & 0xFFFFu] = r;
}

// N1: op-stream evaluator.
__global__ void __launch_bounds__(512, 2) rtl_eval_kernel(const EvalParams p) {
  extern __shared__ uint32_t sm[];
  const uint32_t lane = threadIdx.x & 31u, wl = threadIdx.x >> 5;
  const uint32_t tile = blockIdx.x;
  const uint32_t s = tile * 32u + lane;
  const uint32_t N = p.N_pad, N32 = p.N_pad >> 5;
  const uint32_t nthr = blockDim.x;
  // per-warp descriptor staging buffer: 32 descriptors (512 B), refilled from
  // registers that were prefetched while the previous chunk executed
  uint4 *dbuf = reinterpret_cast<uint4 *>(sm + p.desc_smem_off) + wl * 32u;
  uint4 pf = make_uint4(0, 0, 0, 0);
  uint32_t pf_k = 0xFFFFFFFFu;
  // bit-sliced ops: one per thread per step, prefetched one step ahead
  uint4 pfb = make_uint4(0, 0, 0, 0);
  {
    const uint32_t b0 = __ldg(p.bit_ptr + p.step_begin), b1 = __ldg(p.bit_ptr + p.step_begin + 1);
    if (b0 + threadIdx.x < b1) pfb = __ldg(p.bitdesc + b0 + threadIdx.x);
  }

  for (uint32_t c = 0; c < p.n_cycles; c++) {
    const uint32_t par = (uint32_t)((p.cycle0 + c) & 1ull);
    const Arena cur = p.state[par], nxt = p.state[par ^ 1u];
    Arena inp;
    inp.bit = p.in.bit + (size_t)c * p.in_stride[CLS_BIT];
    inp.u8 = p.in.u8 + (size_t)c * p.in_stride[CLS_U8];
    inp.u16 = p.in.u16 + (size_t)c * p.in_stride[CLS_U16];
    inp.u32 = p.in.u32 + (size_t)c * p.in_stride[CLS_U32];
    uint32_t *out = p.out + (size_t)c * p.OW * N;
    unsigned long long dig = 0ull;

    for (uint32_t step = p.step_begin; step < p.step_end; step++) {
      const uint32_t kb = __ldg(p.step_ptr + step * p.L + wl);
      const uint32_t ke = __ldg(p.step_ptr + step * p.L + wl + 1);
      const uint32_t nstep = step + 1 < p.step_end ? step + 1 : p.step_begin;
      const uint32_t nb = __ldg(p.step_ptr + nstep * p.L + wl);
      // ---- bit-sliced ops of this step (lane = op)
      {
        const uint32_t bb = __ldg(p.bit_ptr + step), be = __ldg(p.bit_ptr + step + 1);
        const uint32_t nbb = __ldg(p.bit_ptr + nstep), nbe = __ldg(p.bit_ptr + nstep + 1);
        const uint4 qb = pfb;
        if (nbb + threadIdx.x < nbe) pfb = __ldg(p.bitdesc + nbb + threadIdx.x);
        if (bb + threadIdx.x < be) exec_bit(sm, qb);
        for (uint32_t k = bb + threadIdx.x + nthr; k < be; k += nthr) exec_bit(sm, __ldg(p.bitdesc + k));
      }
      // ---- this warp's list of per-stimulus ops
      for (uint32_t k0 = kb; k0 < ke; k0 += 32u) {
        if (pf_k != k0) pf = __ldg(p.desc + k0 + lane);
        __syncwarp();
        dbuf[lane] = pf;
        __syncwarp();
        pf_k = (k0 + 32u < ke) ? k0 + 32u : nb;
        pf = __ldg(p.desc + pf_k + lane);   // the array is padded by 32 descriptors
        const uint32_t nk = min(32u, ke - k0);
        for (uint32_t j = 0; j < nk; j++) {
          const uint4 q = dbuf[j];
          const uint32_t code = q.x & 0xFFu;
          if (code < 32u) {   // narrow compute op
            const uint32_t hid = (q.w >> 13) & 31u;
            if (hid) {   // specialized handler: uniform operand layout, one small op switch
              fast_narrow(sm, q, hid, code, lane);
              continue;
            }
            const uint32_t x = fetch1(sm, q.y >> 16, (q.x >> 8) & 7u, lane);
            const uint32_t y = (q.w & (1u << 11)) ? fetch1(sm, q.z & 0xFFFFu, (q.x >> 11) & 7u, lane) : 0u;
            const uint32_t z = (q.w & (1u << 12)) ? fetch1(sm, q.z >> 16, (q.x >> 14) & 7u, lane) : 0u;
            const uint32_t wd = (q.x >> 20) & 63u;
            const uint32_t r = alu1(code, x, y, z, wd, q.x >> 26, q.w & 63u, (q.w >> 6) & 31u) &
                               (0xFFFFFFFFu >> (32u - wd));
            store1(sm, q.y & 0xFFFFu, (q.x >> 17) & 7u, r, lane);
            continue;
          }
          if (code == CODE_WIDE) {
            exec_wide(sm, p.wide + q.y, lane);
            continue;
          }
          const uint32_t cls = (q.x >> 8) & 3u, nw = (q.x >> 12) & 63u;
          switch (code) {
            case CODE_LD_REG: ld_class(sm, q.y, cls, nw, cur, q.z, N, tile, lane); break;
            case CODE_LD_X: ld_class(sm, q.y, cls, nw, p.xnet, q.z, N, tile, lane); break;
            case CODE_LD_IN: ld_class(sm, q.y, cls, nw, inp, q.z, N, tile, lane); break;
            case CODE_LD_CONST:
              if ((q.x >> 18) & 1u) {   // broadcast copy
                if (lane < nw) sm[q.y + lane] = __ldg(p.consts + q.z + lane);
              } else {
                #pragma unroll 1
                for (uint32_t i = 0; i < nw; i++) sm[q.y + 32u * i + lane] = __ldg(p.consts + q.z + i);
              }
              break;
            case CODE_ST_REG:
            case CODE_ST_X: {
              const Arena ar = code == CODE_ST_REG ? nxt : p.xnet;
              const bool dg = p.digest && code == CODE_ST_REG;
              const uint32_t row = q.z, aux = q.w, a = q.y;
              if (cls == CLS_BIT) {
                const uint32_t word = sm[a];
                if (lane == 0) ar.bit[(size_t)row * N32 + tile] = word;
                if (dg) dig ^= mix64(((unsigned long long)(aux + 1u + 0x80000000u) << 32) | ((word >> lane) & 1u));
              } else if (cls == CLS_U32) {
                #pragma unroll 1
                for (uint32_t i = 0; i < nw; i++) {
                  const uint32_t v = sm[a + 32u * i + lane];
                  ar.u32[(size_t)(row + i) * N + s] = v;
                  if (dg) dig ^= mix64(((unsigned long long)(aux + i + 1u + 0x80000000u) << 32) | v);
                }
              } else {
                // 32 byte / half-word lanes: copy the packed words (8 or 16 lanes)
                const uint32_t nlw = cls == CLS_U8 ? 8u : 16u;
                uint8_t *dst = cls == CLS_U8 ? ar.u8 + (size_t)row * N + tile * 32u
                                             : reinterpret_cast<uint8_t *>(ar.u16 + (size_t)row * N + tile * 32u);
                if (lane < nlw) reinterpret_cast<uint32_t *>(dst)[lane] = sm[a + lane];
                if (dg) {
                  const uint32_t v = cls == CLS_U8 ? reinterpret_cast<const uint8_t *>(sm)[4u * a + lane]
                                                   : reinterpret_cast<const uint16_t *>(sm)[2u * a + lane];
                  dig ^= mix64(((unsigned long long)(aux + 1u + 0x80000000u) << 32) | v);
                }
              }
              break;
            }
            case CODE_ST_OUT: {
              const uint32_t lay = (q.x >> 18) & 7u, a = q.y;
              #pragma unroll 1
              for (uint32_t i = 0; i < nw; i++) {
                const uint32_t v = lay == LC_U32 ? sm[a + 32u * i + lane] : fetch1(sm, a, lay, lane);
                out[(size_t)(q.z + i) * N + s] = v;
                if (p.digest) dig ^= mix64(((unsigned long long)(q.z + i + 1u) << 32) | v);
              }
              break;
            }
            default:
              break;
          }
        }
      }
      // loads were issued up to load-ahead steps early: wait until only the
      // groups the compiler allows are still pending (program.h step_wait)
      asm volatile("cp.async.commit_group;" ::: "memory");
      switch (__ldg(p.step_wait + step)) {
        case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
        case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
        case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
        default: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
      }
      __syncthreads();
    }
    if (p.digest && dig) atomicXor(p.digest + (size_t)c * N + s, dig);
  }
}

// The attribute is process-wide per kernel: set it to the device's opt-in
// maximum (not the size of the context loaded last), so a context needing more
// shared memory than one loaded after it still launches.
cudaError_t eval_set_smem(uint32_t /*smem_bytes*/) {
  int dev = 0, optin = 232448;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return cudaFuncSetAttribute(rtl_eval_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
}

cudaError_t launch_eval(const EvalParams &p, uint32_t smem_bytes, cudaStream_t st) {
  dim3 grid(p.N_pad / 32u), block(32u * p.L);
  rtl_eval_kernel<<<grid, block, smem_bytes, st>>>(p);
  return cudaGetLastError();
}

// ------------------------------------------------------------ N2 / N3 --
// N2: stimulus chunk [N][nc][IW] (user layout, row pitch src_pitch words) ->
// per-cycle class-formatted input rows (packed bits / u8 / u16 / u32 word
// rows, [nc][rows][N]) through a 32x32 shared-memory transpose, masking the
// bits above each input's width (reading 15). Stimuli >= N read as zero.
__global__ void stim_transpose_kernel(const uint32_t *__restrict__ src, uint64_t src_pitch, uint32_t N,
                                      uint32_t nc, uint32_t IW, const uint32_t *__restrict__ mask,
                                      const RegWord *__restrict__ map, Arena dst, InStride st,
                                      uint32_t N_pad) {
  __shared__ uint32_t t[32][33];
  const uint32_t cols = nc * IW;                       // (cycle, word) pairs
  const uint32_t j0 = blockIdx.x * 32u, s0 = blockIdx.y * 32u;
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t s = s0 + r, j = j0 + threadIdx.x;
    uint32_t v = 0;
    if (s < N && j < cols) v = src[(size_t)s * src_pitch + j] & __ldg(mask + (j % IW));
    t[r][threadIdx.x] = v;
  }
  __syncthreads();
  const uint32_t lane = threadIdx.x;
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t j = j0 + r, s = s0 + lane;
    if (j >= cols) continue;                           // warp-uniform
    const uint32_t c = j / IW, k = j % IW;
    const RegWord m = map[k];
    const uint32_t v = t[lane][r];
    switch (m.cls) {
      case CLS_BIT: {
        const uint32_t bits = __ballot_sync(0xFFFFFFFFu, v & 1u);
        if (lane == 0) dst.bit[(size_t)c * st.s[CLS_BIT] + (size_t)m.row * (N_pad >> 5) + (s0 >> 5)] = bits;
        break;
      }
      case CLS_U8: dst.u8[(size_t)c * st.s[CLS_U8] + (size_t)m.row * N_pad + s] = (uint8_t)v; break;
      case CLS_U16: dst.u16[(size_t)c * st.s[CLS_U16] + (size_t)m.row * N_pad + s] = (uint16_t)v; break;
      default: dst.u32[(size_t)c * st.s[CLS_U32] + (size_t)m.row * N_pad + s] = v; break;
    }
  }
}

cudaError_t launch_stim_transpose(const uint32_t *src, uint64_t src_pitch, uint32_t N, uint32_t N_pad,
                                  uint32_t nc, uint32_t IW, const uint32_t *mask, const RegWord *map,
                                  Arena dst, InStride st, cudaStream_t stream) {
  if (nc == 0 || IW == 0) return cudaSuccess;
  dim3 grid((nc * IW + 31u) / 32u, N_pad / 32u), block(32, 8);
  stim_transpose_kernel<<<grid, block, 0, stream>>>(src, src_pitch, N, nc, IW, mask, map, dst, st, N_pad);
  return cudaGetLastError();
}

__global__ void out_transpose_kernel(const uint32_t *__restrict__ src, uint32_t N, uint32_t N_pad,
                                     uint32_t cols, uint32_t *__restrict__ dst, uint64_t dst_pitch) {
  __shared__ uint32_t t[32][33];
  const uint32_t j0 = blockIdx.x * 32u, s0 = blockIdx.y * 32u;
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t j = j0 + r, s = s0 + threadIdx.x;
    t[r][threadIdx.x] = (j < cols && s < N_pad) ? src[(size_t)j * N_pad + s] : 0u;
  }
  __syncthreads();
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t s = s0 + r, j = j0 + threadIdx.x;
    if (s < N && j < cols) dst[(size_t)s * dst_pitch + j] = t[threadIdx.x][r];
  }
}

cudaError_t launch_out_transpose(const uint32_t *src, uint32_t N, uint32_t N_pad, uint32_t nc,
                                 uint32_t OW, uint32_t *dst, uint64_t dst_pitch, cudaStream_t st) {
  if (nc == 0 || OW == 0) return cudaSuccess;
  dim3 grid((nc * OW + 31u) / 32u, N_pad / 32u), block(32, 8);
  out_transpose_kernel<<<grid, block, 0, st>>>(src, N, N_pad, nc * OW, dst, dst_pitch);
  return cudaGetLastError();
}

__global__ void digest_transpose_kernel(const unsigned long long *__restrict__ src, uint32_t N,
                                        uint32_t N_pad, uint32_t nc, unsigned long long *__restrict__ dst,
                                        uint64_t dst_pitch) {
  __shared__ unsigned long long t[32][33];
  const uint32_t j0 = blockIdx.x * 32u, s0 = blockIdx.y * 32u;
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t j = j0 + r, s = s0 + threadIdx.x;
    t[r][threadIdx.x] = (j < nc && s < N_pad) ? src[(size_t)j * N_pad + s] : 0ull;
  }
  __syncthreads();
  for (uint32_t r = threadIdx.y; r < 32u; r += blockDim.y) {
    const uint32_t s = s0 + r, j = j0 + threadIdx.x;
    if (s < N && j < nc) dst[(size_t)s * dst_pitch + j] = t[threadIdx.x][r];
  }
}

cudaError_t launch_digest_transpose(const unsigned long long *src, uint32_t N, uint32_t N_pad, uint32_t nc,
                                    unsigned long long *dst, uint64_t dst_pitch, cudaStream_t st) {
  if (nc == 0) return cudaSuccess;
  dim3 grid((nc + 31u) / 32u, N_pad / 32u), block(32, 8);
  digest_transpose_kernel<<<grid, block, 0, st>>>(src, N, N_pad, nc, dst, dst_pitch);
  return cudaGetLastError();
}

// ----------------------------------------------------------------- N4 --
// one warp per (register word, 32-stimulus tile)
__global__ void regs_import_kernel(const uint32_t *__restrict__ src, uint64_t src_stride,
                                   const RegWord *__restrict__ map, uint32_t RW, uint32_t N,
                                   uint32_t N_pad, Arena a) {
  const uint32_t k = blockIdx.x;
  const uint32_t s = blockIdx.y * blockDim.x + threadIdx.x;
  if (s >= N_pad) return;
  const uint32_t lane = threadIdx.x & 31u;
  const RegWord m = map[k];
  const uint32_t si = s < N ? s : (N ? N - 1 : 0);   // padding stimuli mirror the last one
  const uint32_t v = src[(size_t)si * src_stride + k];
  switch (m.cls) {
    case CLS_BIT: {
      const uint32_t bits = __ballot_sync(0xFFFFFFFFu, v & 1u);
      if (lane == 0) a.bit[(size_t)m.row * (N_pad >> 5) + (s >> 5)] = bits;
      break;
    }
    case CLS_U8: a.u8[(size_t)m.row * N_pad + s] = (uint8_t)v; break;
    case CLS_U16: a.u16[(size_t)m.row * N_pad + s] = (uint16_t)v; break;
    default: a.u32[(size_t)m.row * N_pad + s] = v; break;
  }
}

cudaError_t launch_regs_import(const uint32_t *src, uint64_t src_stride, const RegWord *map, uint32_t RW,
                               uint32_t N, uint32_t N_pad, Arena a, cudaStream_t st) {
  if (RW == 0) return cudaSuccess;
  dim3 grid(RW, N_pad / 256u + ((N_pad % 256u) ? 1u : 0u)), block(256);
  regs_import_kernel<<<grid, block, 0, st>>>(src, src_stride, map, RW, N, N_pad, a);
  return cudaGetLastError();
}

__global__ void regs_export_kernel(Arena a, const RegWord *__restrict__ map, uint32_t RW, uint32_t N,
                                   uint32_t N_pad, uint32_t *__restrict__ dst) {
  const uint32_t k = blockIdx.x;
  const uint32_t s = blockIdx.y * blockDim.x + threadIdx.x;
  if (s >= N) return;
  const RegWord m = map[k];
  uint32_t v;
  switch (m.cls) {
    case CLS_BIT: v = (a.bit[(size_t)m.row * (N_pad >> 5) + (s >> 5)] >> (s & 31u)) & 1u; break;
    case CLS_U8: v = a.u8[(size_t)m.row * N_pad + s]; break;
    case CLS_U16: v = a.u16[(size_t)m.row * N_pad + s]; break;
    default: v = a.u32[(size_t)m.row * N_pad + s]; break;
  }
  dst[(size_t)s * RW + k] = v;
}

cudaError_t launch_regs_export(Arena a, const RegWord *map, uint32_t RW, uint32_t N, uint32_t N_pad,
                               uint32_t *dst, cudaStream_t st) {
  if (RW == 0 || N == 0) return cudaSuccess;
  dim3 grid(RW, (N + 255u) / 256u), block(256);
  regs_export_kernel<<<grid, block, 0, st>>>(a, map, RW, N, N_pad, dst);
  return cudaGetLastError();
}


// ------------------------------------------------------------- N5 / digest --
// N5 toggle coverage of one cycle: for register word k (class row m.row),
// cov[k] |= OR over the real stimuli s < N of (R_c[s][k] ^ R_{c+1}[s][k]).
// Grid (RW, stimulus chunks): each thread ORs 32-bit words of the two
// arenas' rows (4 / 2 / 1 stimuli per word for u8 / u16 / u32 rows, 32 for
// packed bit rows), padding stimuli masked out; a warp OR-reduction, then
// one atomicOr per warp (ballot / reduce + atomicOr, NS subsystem 4).
__global__ void toggle_coverage_kernel(Arena cur, Arena nxt, const RegWord *__restrict__ map, uint32_t N,
                                       uint32_t N_pad, uint32_t *__restrict__ cov) {
  const uint32_t k = blockIdx.x;
  const RegWord m = map[k];
  const uint32_t per = m.cls == CLS_BIT ? 32u : m.cls == CLS_U8 ? 4u : m.cls == CLS_U16 ? 2u : 1u;
  const uint32_t words = N_pad / per;   // 32-bit words of the row
  const uint32_t *a, *b;
  switch (m.cls) {
    case CLS_BIT: a = cur.bit + (size_t)m.row * (N_pad >> 5); b = nxt.bit + (size_t)m.row * (N_pad >> 5); break;
    case CLS_U8: a = (const uint32_t *)(cur.u8 + (size_t)m.row * N_pad); b = (const uint32_t *)(nxt.u8 + (size_t)m.row * N_pad); break;
    case CLS_U16: a = (const uint32_t *)(cur.u16 + (size_t)m.row * N_pad); b = (const uint32_t *)(nxt.u16 + (size_t)m.row * N_pad); break;
    default: a = cur.u32 + (size_t)m.row * N_pad; b = nxt.u32 + (size_t)m.row * N_pad; break;
  }
  uint32_t acc = 0;
  for (uint32_t i = blockIdx.y * blockDim.x + threadIdx.x; i < words; i += gridDim.y * blockDim.x) {
    uint32_t t = __ldg(a + i) ^ __ldg(b + i);
    const uint32_t s0 = i * per;                  // first stimulus of this word
    if (s0 + per > N) {                           // mask the padding stimuli
      const uint32_t real = s0 >= N ? 0u : N - s0;
      const uint32_t bits_per = 32u / per;
      t &= real * bits_per >= 32u ? 0xFFFFFFFFu : ((1u << (real * bits_per)) - 1u);
    }
    if (m.cls == CLS_BIT) t = t ? 1u : 0u;        // a 1-bit register: bit 0 toggled
    else if (per > 1) {                           // fold the stimulus lanes of the word
      const uint32_t lb = 32u / per;
      uint32_t f = 0;
      for (uint32_t j = 0; j < per; j++) f |= (t >> (j * lb)) & ((1u << lb) - 1u);
      t = f;
    }
    acc |= t;
  }
  acc = __reduce_or_sync(0xFFFFFFFFu, acc);
  if ((threadIdx.x & 31u) == 0 && acc) atomicOr(cov + k, acc);
}

cudaError_t launch_toggle_coverage(Arena cur, Arena nxt, const RegWord *map, uint32_t RW, uint32_t N,
                                   uint32_t N_pad, uint32_t *cov, cudaStream_t st) {
  if (RW == 0 || N == 0) return cudaSuccess;
  const uint32_t chunks = std::min<uint32_t>(64u, (N_pad + 8191u) / 8192u);
  toggle_coverage_kernel<<<dim3(RW, chunks), 256, 0, st>>>(cur, nxt, map, N, N_pad, cov);
  return cudaGetLastError();
}

__device__ __forceinline__ uint64_t mix64_dev(uint64_t z) {   // splitmix64 finalizer (DIGEST)
  z ^= z >> 30;
  z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27;
  z *= 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Per-stimulus DIGEST of the register state (the register part of the
// per-cycle digest): dig[s] = XOR_k mix(((k+1+2^31) << 32) | R[s][k]).
// One thread per stimulus walks the RW words; consecutive threads read
// consecutive stimuli of a row (coalesced).
__global__ void reg_digest_kernel(Arena a, const RegWord *__restrict__ map, uint32_t RW, uint32_t N,
                                  uint32_t N_pad, unsigned long long *__restrict__ dig) {
  const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= N) return;
  uint64_t h = 0;
  for (uint32_t k = 0; k < RW; k++) {
    const RegWord m = map[k];
    uint32_t v;
    switch (m.cls) {
      case CLS_BIT: v = (a.bit[(size_t)m.row * (N_pad >> 5) + (s >> 5)] >> (s & 31u)) & 1u; break;
      case CLS_U8: v = a.u8[(size_t)m.row * N_pad + s]; break;
      case CLS_U16: v = a.u16[(size_t)m.row * N_pad + s]; break;
      default: v = a.u32[(size_t)m.row * N_pad + s]; break;
    }
    h ^= mix64_dev(((uint64_t)(k + 1u + 0x80000000u) << 32) | v);
  }
  dig[s] = h;
}

cudaError_t launch_reg_digest(Arena a, const RegWord *map, uint32_t RW, uint32_t N, uint32_t N_pad,
                              unsigned long long *dig, cudaStream_t st) {
  if (N == 0) return cudaSuccess;
  reg_digest_kernel<<<(N + 255u) / 256u, 256, 0, st>>>(a, map, RW, N, N_pad, dig);
  return cudaGetLastError();
}

// ------------------------------------------------------------ memories --
// Memory write ports at the clock edge (reading 12): after the
// cycle's partitions stored every port's (address, data, enable) words in the
// port arena, one thread per stimulus applies the ports in order (a later port
// wins): entry V[addr] := V[data] zero-extended / truncated to the memory
// width when V[en] != 0 and V[addr] < depth. Memory rows are [row][N_pad] u32.
__global__ void mem_commit_kernel(uint32_t *__restrict__ mem, const uint32_t *__restrict__ port,
                                  const MemPortDev *__restrict__ ports, uint32_t n_ports, uint32_t N,
                                  uint32_t N_pad) {
  const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= N) return;
  for (uint32_t p = 0; p < n_ports; p++) {
    const MemPortDev P = ports[p];
    uint32_t en = 0;
    for (uint32_t t = 0; t < (P.en_width + 31u) / 32u; t++) en |= port[(size_t)(P.en_word + t) * N_pad + s];
    if (!en) continue;
    const uint32_t idx = port[(size_t)P.addr_word * N_pad + s];
    if (idx >= P.depth) continue;
    const uint32_t nwm = (P.width + 31u) / 32u, nwd = (P.data_width + 31u) / 32u;
    for (uint32_t t = 0; t < nwm; t++) {
      uint32_t v = t < nwd ? port[(size_t)(P.data_word + t) * N_pad + s] : 0u;
      if (t == nwm - 1 && (P.width & 31u)) v &= (1u << (P.width & 31u)) - 1u;
      mem[(size_t)(P.row0 + idx * nwm + t) * N_pad + s] = v;
    }
  }
}

cudaError_t launch_mem_commit(uint32_t *mem, const uint32_t *port, const MemPortDev *ports, uint32_t n_ports,
                              uint32_t N, uint32_t N_pad, cudaStream_t st) {
  if (!n_ports || !N) return cudaSuccess;
  mem_commit_kernel<<<(N + 255u) / 256u, 256, 0, st>>>(mem, port, ports, n_ports, N, N_pad);
  return cudaGetLastError();
}

// memory rows <- their initial values (the same for every stimulus)
__global__ void mem_init_kernel(uint32_t *__restrict__ mem, const uint32_t *__restrict__ init, uint32_t N_pad) {
  const uint32_t r = blockIdx.y;
  const uint32_t v = init[r];
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < N_pad; s += gridDim.x * blockDim.x)
    mem[(size_t)r * N_pad + s] = v;
}

cudaError_t launch_mem_init(uint32_t *mem, const uint32_t *init, uint32_t MR, uint32_t N_pad, cudaStream_t st) {
  if (!MR) return cudaSuccess;
  mem_init_kernel<<<dim3(std::min<uint32_t>(64u, (N_pad + 255u) / 256u), MR), 256, 0, st>>>(mem, init, N_pad);
  return cudaGetLastError();
}

// memory rows [MR][N_pad] -> dst [N][MR]
__global__ void mem_export_kernel(const uint32_t *__restrict__ mem, uint32_t MR, uint32_t N, uint32_t N_pad,
                                  uint32_t *__restrict__ dst) {
  const uint32_t r = blockIdx.y;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < N; s += gridDim.x * blockDim.x)
    dst[(size_t)s * MR + r] = mem[(size_t)r * N_pad + s];
}

cudaError_t launch_mem_export(const uint32_t *mem, uint32_t MR, uint32_t N, uint32_t N_pad, uint32_t *dst,
                              cudaStream_t st) {
  if (!MR || !N) return cudaSuccess;
  mem_export_kernel<<<dim3(std::min<uint32_t>(64u, (N + 255u) / 256u), MR), 256, 0, st>>>(mem, MR, N, N_pad, dst);
  return cudaGetLastError();
}

// ====================================================================== v4 --
// Run-based evaluator over the lowered micro-op stream (lower.cpp). Same tile
// / op-lane / step structure as rtl_eval_kernel; each op-lane warp walks its
// runs (program.h G_* groups) and executes each in an unrolled loop whose
// operand loads are all issued before any store (ops of one step are
// independent and never share a slot). Micro-ops are read straight from
// global memory (warp-uniform 16-byte loads, L1 / L2 resident; the next
// step's block is prefetched into L1). One handler per group keeps the whole
// hot loop small: like the JIT kernels, an evaluator whose code does not fit
// the instruction cache is instruction-fetch bound.
namespace v4 {

template <int E>
__device__ __forceinline__ uint32_t lde(const uint8_t *p) {
  if constexpr (E == 1) return *p;
  else if constexpr (E == 2) return *reinterpret_cast<const uint16_t *>(p);
  else return *reinterpret_cast<const uint32_t *>(p);
}
template <int E>
__device__ __forceinline__ void ste(uint8_t *p, uint32_t v) {
  if constexpr (E == 1) *p = (uint8_t)v;
  else if constexpr (E == 2) *reinterpret_cast<uint16_t *>(p) = (uint16_t)v;
  else *reinterpret_cast<uint32_t *>(p) = v;
}
__device__ __forceinline__ uint32_t lds32(const uint8_t *p) { return *reinterpret_cast<const uint32_t *>(p); }
__device__ __forceinline__ void sts32(uint8_t *p, uint32_t v) { *reinterpret_cast<uint32_t *>(p) = v; }

constexpr int UNR = (int)kUnroll;   // runs of these groups are padded to a multiple (lower.cpp)

// AND / OR / XOR: ((a & b & A) | ((a ^ b) & B)) & mask
template <int E>
__device__ __forceinline__ void h_log(const uint4 *__restrict__ u, uint32_t n, uint8_t *base, uint32_t A, uint32_t B) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t x[UNR], y[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      x[k] = lde<E>(base + q[k].y);
      y[k] = lde<E>(base + q[k].z);
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) ste<E>(base + q[k].x, ((x[k] & y[k] & A) | ((x[k] ^ y[k]) & B)) & q[k].w);
  }
}

// ADD / SUB: (a + (b ^ S) + C) & mask
template <int E>
__device__ __forceinline__ void h_ari(const uint4 *__restrict__ u, uint32_t n, uint8_t *base, uint32_t S, uint32_t C) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t x[UNR], y[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      x[k] = lde<E>(base + q[k].y);
      y[k] = lde<E>(base + q[k].z);
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) ste<E>(base + q[k].x, (x[k] + (y[k] ^ S) + C) & q[k].w);
  }
}

// COPY / NOT / SLICE: ((a >> z) ^ INV) & mask
template <int E>
__device__ __forceinline__ void h_un(const uint4 *__restrict__ u, uint32_t n, uint8_t *base, uint32_t INV) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t x[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) x[k] = lde<E>(base + q[k].y);
#pragma unroll
    for (int k = 0; k < UNR; k++) ste<E>(base + q[k].x, ((x[k] >> q[k].z) ^ INV) & q[k].w);
  }
}

// MUX on a 1-bit select: {d | ms << 24, sel, t, e}
template <int E>
__device__ __forceinline__ void h_mux(const uint4 *__restrict__ u, uint32_t n, uint8_t *base, uint8_t *smb,
                                      uint32_t lane) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t sl[UNR], t[UNR], e[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      sl[k] = lds32(smb + q[k].y);
      t[k] = lde<E>(base + q[k].z);
      e[k] = lde<E>(base + q[k].w);
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      const uint32_t r = ((sl[k] >> lane) & 1u) ? t[k] : e[k];
      ste<E>(base + (q[k].x & 0xFFFFFFu), r & (0xFFFFFFFFu >> (q[k].x >> 24)));
    }
  }
}

// unsigned compare -> packed 1-bit result, cc = EQ NE LTU LEU GTU GEU
__device__ __forceinline__ bool cmp_cc(uint32_t cc, uint32_t x, uint32_t y) {
  // relation index 0: x > y, 1: x == y, 2: x < y; per cc the set of indices
  // where it holds: EQ 010, NE 101, LTU 100, LEU 110, GTU 001, GEU 011
  const uint32_t i = x < y ? 2u : (x == y ? 1u : 0u);
  return (0x316452u >> (4u * cc + i)) & 1u;
}
template <int E>
__device__ __forceinline__ void h_cmp(const uint4 *__restrict__ u, uint32_t n, uint8_t *base, uint8_t *smb,
                                      uint32_t lane, uint32_t cc) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t x[UNR], y[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      x[k] = lde<E>(base + q[k].y);
      y[k] = lde<E>(base + q[k].z);
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      const uint32_t bits = __ballot_sync(0xFFFFFFFFu, cmp_cc(cc, x[k], y[k]));
      if (lane == 0) sts32(smb + q[k].x, bits);
    }
  }
}

// word: (fshr(lo, hi, sh) | z) & (~0 >> ms) : {d | ms << 24, lo, hi, z | sh << 24}
__device__ __forceinline__ void h_fun(const uint4 *__restrict__ u, uint32_t n, uint8_t *b4) {
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t lo[UNR], hi[UNR], z[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      lo[k] = lds32(b4 + q[k].y);
      hi[k] = lds32(b4 + q[k].z);
      z[k] = lds32(b4 + (q[k].w & 0xFFFFFFu));
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      const uint32_t r = (__funnelshift_r(lo[k], hi[k], q[k].w >> 24) | z[k]) & (0xFFFFFFFFu >> (q[k].x >> 24));
      sts32(b4 + (q[k].x & 0xFFFFFFu), r);
    }
  }
}

// word stores of a constant: every lane (per-lane row) or broadcast word
__device__ __forceinline__ void h_const(const uint4 *__restrict__ u, uint32_t n, uint8_t *p) {
  uint4 qn = __ldg(u);
  for (uint32_t i = 0; i < n; i++) {
    const uint4 q = qn;
    if (i + 1 < n) qn = __ldg(u + i + 1);   // next micro-op in flight
    sts32(p + q.x, q.y);
  }
}

// wide add / sub / neg: {d, a, b, nd | na<<6 | nb<<12 | sub<<18 | ms<<24}
__device__ __forceinline__ void h_wadd(const uint4 *__restrict__ u, uint32_t n, uint8_t *b4) {
  uint4 qn = __ldg(u);
  for (uint32_t j = 0; j < n; j++) {
    const uint4 q = qn;
    if (j + 1 < n) qn = __ldg(u + j + 1);   // next micro-op in flight
    const uint32_t nd = q.w & 63u, na = (q.w >> 6) & 63u, nb = (q.w >> 12) & 63u, sub = (q.w >> 18) & 1u;
    const uint32_t S = 0u - sub;
    uint32_t carry = sub;
    for (uint32_t i = 0; i < nd; i++) {
      const uint32_t x = i < na ? lds32(b4 + q.y + 128u * i) : 0u;
      const uint32_t y = (i < nb ? lds32(b4 + q.z + 128u * i) : 0u) ^ S;
      const unsigned long long t = (unsigned long long)x + y + carry;
      carry = (uint32_t)(t >> 32);
      uint32_t r = (uint32_t)t;
      if (i == nd - 1) r &= 0xFFFFFFFFu >> (q.w >> 24);
      sts32(b4 + q.x + 128u * i, r);
    }
  }
}

// wide unsigned compare -> 1 bit: {d, a, b, n | na<<6 | nb<<12 | cc<<18}
__device__ __forceinline__ void h_wcmp(const uint4 *__restrict__ u, uint32_t n, uint8_t *b4, uint8_t *smb,
                                       uint32_t lane) {
  uint4 qn = __ldg(u);
  for (uint32_t j = 0; j < n; j++) {
    const uint4 q = qn;
    if (j + 1 < n) qn = __ldg(u + j + 1);   // next micro-op in flight
    const uint32_t nw = q.w & 63u, na = (q.w >> 6) & 63u, nb = (q.w >> 12) & 63u, cc = (q.w >> 18) & 7u;
    uint32_t rel = 1u;   // 0: a > b, 1: equal, 2: a < b (most significant differing word)
    for (int i = (int)nw - 1; i >= 0 && rel == 1u; i--) {
      const uint32_t x = (uint32_t)i < na ? lds32(b4 + q.y + 128u * i) : 0u;
      const uint32_t y = (uint32_t)i < nb ? lds32(b4 + q.z + 128u * i) : 0u;
      rel = x < y ? 2u : (x == y ? 1u : 0u);
    }
    const uint32_t bits = __ballot_sync(0xFFFFFFFFu, (0x316452u >> (4u * cc + rel)) & 1u);
    if (lane == 0) sts32(smb + q.x, bits);
  }
}

__device__ __forceinline__ void cp_async16(uint8_t *smem_dst, const void *gsrc) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}

__device__ __forceinline__ uint8_t *arena_ptr(const Arena &a, uint32_t cls) {
  return cls == CLS_BIT ? reinterpret_cast<uint8_t *>(a.bit)
                        : cls == CLS_U8 ? a.u8 : cls == CLS_U16 ? reinterpret_cast<uint8_t *>(a.u16)
                                                                : reinterpret_cast<uint8_t *>(a.u32);
}

// row loads {slot, row}: a bit row is one word of the tile (one lane per
// row); u8 / u16 / u32 row segments are 32 / 64 / 128 bytes, 16 bytes per
// lane (2 / 4 / 8 lanes per row)
__device__ __forceinline__ void h_ld(const uint4 *__restrict__ u, uint32_t n, uint8_t *ar, uint32_t cls, size_t N,
                                     uint32_t tile, uint32_t lane, uint8_t *smb) {
  if (cls == CLS_BIT) {
    const size_t rs = N >> 3;
    for (uint32_t j = lane; j < n; j += 32u) {
      const uint4 q = __ldg(u + j);
      cp_async4(smb + q.x, ar + (size_t)q.y * rs + 4u * tile);
    }
    return;
  }
  const uint32_t sh = cls, part = lane & ((1u << sh) - 1u);
  const size_t rs = N << (sh - 1u);
  const uint32_t tb = (16u << sh) * tile + 16u * part;
  for (uint32_t j = lane >> sh; j < n; j += (32u >> sh)) {
    const uint4 q = __ldg(u + j);
    cp_async16(smb + q.x + 16u * part, ar + (size_t)q.y * rs + tb);
  }
}

// row stores {slot, row, reg word}; with the digest (check mode) one row at
// a time, lane = stimulus
template <bool DIG>
__device__ __forceinline__ void h_st(const uint4 *__restrict__ u, uint32_t n, uint8_t *ar, uint32_t cls, size_t N,
                                     uint32_t tile, uint32_t lane, uint8_t *smb, bool dg, unsigned long long &dig) {
  if (DIG && dg) {
    for (uint32_t j = 0; j < n; j++) {
      const uint4 q = __ldg(u + j);
      uint32_t v;
      if (cls == CLS_BIT) {
        const uint32_t w = lds32(smb + q.x);
        if (lane == 0) reinterpret_cast<uint32_t *>(ar)[(size_t)q.y * (N >> 5) + tile] = w;
        v = (w >> lane) & 1u;
      } else if (cls == CLS_U8) {
        v = smb[q.x + lane];
        ar[(size_t)q.y * N + tile * 32u + lane] = (uint8_t)v;
      } else if (cls == CLS_U16) {
        v = reinterpret_cast<const uint16_t *>(smb + q.x)[lane];
        reinterpret_cast<uint16_t *>(ar)[(size_t)q.y * N + tile * 32u + lane] = (uint16_t)v;
      } else {
        v = lds32(smb + q.x + 4u * lane);
        reinterpret_cast<uint32_t *>(ar)[(size_t)q.y * N + tile * 32u + lane] = v;
      }
      dig ^= mix64(((unsigned long long)(q.z + 1u + 0x80000000u) << 32) | v);
    }
    return;
  }
  if (cls == CLS_BIT) {
    const size_t rs = N >> 3;
    for (uint32_t j = lane; j < n; j += 32u) {
      const uint4 q = __ldg(u + j);
      *reinterpret_cast<uint32_t *>(ar + (size_t)q.y * rs + 4u * tile) = lds32(smb + q.x);
    }
    return;
  }
  const uint32_t sh = cls, part = lane & ((1u << sh) - 1u);
  const size_t rs = N << (sh - 1u);
  const uint32_t tb = (16u << sh) * tile + 16u * part;
  for (uint32_t j = lane >> sh; j < n; j += (32u >> sh)) {
    const uint4 q = __ldg(u + j);
    *reinterpret_cast<uint4 *>(ar + (size_t)q.y * rs + tb) = *reinterpret_cast<const uint4 *>(smb + q.x + 16u * part);
  }
}

// narrow op of any operand layouts (program.h Desc): branch-free operand
// fetch from the layout's element size, layout-dispatched store
// off: BYTE offset of the slot (or the value of an immediate)
__device__ __forceinline__ uint32_t gfetch(const uint8_t *smb, uint32_t off, uint32_t lay, uint32_t lane) {
  if (lay == LC_IMM) return off;
  const uint32_t lg = (0x3405u >> (4u * lay)) & 15u;   // log2 element bits: U32 5, BIT 0, U16 4, U8 3
  const uint32_t t = lane << lg;
  const uint32_t w = lds32(smb + off + ((t >> 5) << 2));
  return (w >> (t & 31u)) & (0xFFFFFFFFu >> (32u - (1u << lg)));
}
__device__ __forceinline__ void gstore(uint8_t *smb, uint32_t off, uint32_t lay, uint32_t r, uint32_t lane) {
  switch (lay) {
    case LC_U32: sts32(smb + 4u * off + 4u * lane, r); break;
    case LC_BIT: {
      const uint32_t m = __ballot_sync(0xFFFFFFFFu, r & 1u);
      if (lane == 0) sts32(smb + 4u * off, m);
      break;
    }
    case LC_U16: *reinterpret_cast<uint16_t *>(smb + 4u * off + 2u * lane) = (uint16_t)r; break;
    default: smb[4u * off + lane] = (uint8_t)r; break;
  }
}
// any-layout narrow ops {d | la<<18 | lb<<21 | lc<<24 | ms<<27, a, b, c|param | ld<<24}
// F: 0 AND/OR/XOR/ADD/SUB (p = op), 1 COPY/NOT/SLICE (p = inversion), 2 CONCAT,
// 3 MUX, 4 unsigned compare (p = cc)
template <int F>
__device__ __forceinline__ void h_gx(const uint4 *__restrict__ u, uint32_t n, uint8_t *smb, uint32_t lane, uint32_t p) {
  const uint32_t A = (p <= 1u) ? 0xFFFFFFFFu : 0u, B = (p == 1u || p == 2u) ? 0xFFFFFFFFu : 0u;
  const uint32_t S = p == 4u ? 0xFFFFFFFFu : 0u, C = p == 4u ? 1u : 0u;
  const bool arith = p >= 3u;
  for (uint32_t i = 0; i < n; i += UNR) {
    uint4 q[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) q[k] = __ldg(u + i + k);
    uint32_t x[UNR], y[UNR], z[UNR];
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      x[k] = gfetch(smb, q[k].y, (q[k].x >> 18) & 7u, lane);
      if constexpr (F != 1) y[k] = gfetch(smb, q[k].z, (q[k].x >> 21) & 7u, lane);
      if constexpr (F == 3) z[k] = gfetch(smb, q[k].w & 0xFFFFFFu, (q[k].x >> 24) & 7u, lane);
    }
#pragma unroll
    for (int k = 0; k < UNR; k++) {
      uint32_t r;
      if constexpr (F == 0) r = arith ? x[k] + (y[k] ^ S) + C : ((x[k] & y[k] & A) | ((x[k] ^ y[k]) & B));
      else if constexpr (F == 1) r = (x[k] >> (q[k].w & 31u)) ^ p;
      else if constexpr (F == 2) r = (x[k] << (q[k].w & 31u)) | y[k];
      else if constexpr (F == 3) r = x[k] ? y[k] : z[k];
      else r = (0x316452u >> (4u * p + (x[k] < y[k] ? 2u : (x[k] == y[k] ? 1u : 0u)))) & 1u;
      gstore(smb, (q[k].x & 0x3FFFFu) >> 2, q[k].w >> 24, r & (0xFFFFFFFFu >> (q[k].x >> 27)), lane);
    }
  }
}

__device__ __noinline__ void h_mix(const uint4 *__restrict__ u, uint32_t n, uint8_t *smb, uint32_t lane, uint32_t op) {
  uint4 qn = __ldg(u);
  for (uint32_t i = 0; i < n; i++) {
    const uint4 q = qn;
    if (i + 1 < n) qn = __ldg(u + i + 1);   // next micro-op in flight
    auto fo = [](uint32_t off, uint32_t lay) { return lay == LC_IMM ? off : 4u * off; };
    const uint32_t la = (q.x >> 8) & 7u, lb = (q.x >> 11) & 7u, lc = (q.x >> 14) & 7u;
    const uint32_t x = gfetch(smb, fo(q.y >> 16, la), la, lane);
    const uint32_t y = (q.w & (1u << 11)) ? gfetch(smb, fo(q.z & 0xFFFFu, lb), lb, lane) : 0u;
    const uint32_t z = (q.w & (1u << 12)) ? gfetch(smb, fo(q.z >> 16, lc), lc, lane) : 0u;
    const uint32_t wd = (q.x >> 20) & 63u;
    const uint32_t r = alu1(op, x, y, z, wd, q.x >> 26, q.w & 63u, (q.w >> 6) & 31u) & (0xFFFFFFFFu >> (32u - wd));
    gstore(smb, q.y & 0xFFFFu, (q.x >> 17) & 7u, r, lane);
  }
}

struct GenCtx {
  uint32_t *sm;
  Arena cur, nxt, xnet, inp;
  uint32_t *out;
  const uint32_t *consts;
  const WideRec *wide;
  uint32_t N, N32, tile, s, lane;
  bool digest;
};

// the generic descriptor path (program.h Desc), as in rtl_eval_kernel
__device__ __noinline__ void exec_gen(const uint4 *__restrict__ u, uint32_t n, const GenCtx &g,
                                      unsigned long long &dig) {
  uint32_t *sm = g.sm;
  const uint32_t lane = g.lane, N = g.N, tile = g.tile, s = g.s;
  uint4 qn = __ldg(u);
  for (uint32_t j = 0; j < n; j++) {
    const uint4 q = qn;
    if (j + 1 < n) qn = __ldg(u + j + 1);   // next micro-op in flight
    const uint32_t code = q.x & 0xFFu;
    if (code == CODE_WIDE) {
      exec_wide(sm, g.wide + q.y, lane);
      continue;
    }
    const uint32_t cls = (q.x >> 8) & 3u, nw = (q.x >> 12) & 63u;
    switch (code) {
      case CODE_LD_REG: ld_class(sm, q.y, cls, nw, g.cur, q.z, N, tile, lane); break;
      case CODE_LD_X: ld_class(sm, q.y, cls, nw, g.xnet, q.z, N, tile, lane); break;
      case CODE_LD_IN: ld_class(sm, q.y, cls, nw, g.inp, q.z, N, tile, lane); break;
      case CODE_ST_REG:
      case CODE_ST_X: {
        const Arena ar = code == CODE_ST_REG ? g.nxt : g.xnet;
        const bool dg = g.digest && code == CODE_ST_REG;
        const uint32_t row = q.z, aux = q.w, a = q.y;
        if (cls == CLS_BIT) {
          const uint32_t word = sm[a];
          if (lane == 0) ar.bit[(size_t)row * g.N32 + tile] = word;
          if (dg) dig ^= mix64(((unsigned long long)(aux + 1u + 0x80000000u) << 32) | ((word >> lane) & 1u));
        } else if (cls == CLS_U32) {
#pragma unroll 1
          for (uint32_t i = 0; i < nw; i++) {
            const uint32_t v = sm[a + 32u * i + lane];
            ar.u32[(size_t)(row + i) * N + s] = v;
            if (dg) dig ^= mix64(((unsigned long long)(aux + i + 1u + 0x80000000u) << 32) | v);
          }
        } else {
          const uint32_t nlw = cls == CLS_U8 ? 8u : 16u;
          uint8_t *dst = cls == CLS_U8 ? ar.u8 + (size_t)row * N + tile * 32u
                                       : reinterpret_cast<uint8_t *>(ar.u16 + (size_t)row * N + tile * 32u);
          if (lane < nlw) reinterpret_cast<uint32_t *>(dst)[lane] = sm[a + lane];
          if (dg) {
            const uint32_t v = cls == CLS_U8 ? reinterpret_cast<const uint8_t *>(sm)[4u * a + lane]
                                             : reinterpret_cast<const uint16_t *>(sm)[2u * a + lane];
            dig ^= mix64(((unsigned long long)(aux + 1u + 0x80000000u) << 32) | v);
          }
        }
        break;
      }
      case CODE_ST_OUT: {
        const uint32_t lay = (q.x >> 18) & 7u, a = q.y;
#pragma unroll 1
        for (uint32_t i = 0; i < nw; i++) {
          const uint32_t v = lay == LC_U32 ? sm[a + 32u * i + lane] : fetch1(sm, a, lay, lane);
          g.out[(size_t)(q.z + i) * N + s] = v;
          if (g.digest) dig ^= mix64(((unsigned long long)(q.z + i + 1u) << 32) | v);
        }
        break;
      }
      default:
        break;
    }
  }
}

template <bool DIG>
__global__ void __launch_bounds__(512, 1) rtl_eval_v4_kernel(const EvalParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t *sm = reinterpret_cast<uint32_t *>(smem);
  const uint32_t lane = threadIdx.x & 31u, wl = threadIdx.x >> 5;
  const uint32_t tile = blockIdx.x;
  const uint32_t N = p.N_pad;
  const uint32_t nthr = blockDim.x;
  uint8_t *b1 = smem + lane, *b2 = smem + 2u * lane, *b4 = smem + 4u * lane;
  for (uint32_t i = threadIdx.x; i < 32u; i += nthr) sm[p.zero_off + i] = 0u;
  __syncthreads();
  GenCtx g;
  g.sm = sm;
  g.xnet = p.xnet;
  g.consts = p.consts;
  g.wide = p.wide;
  g.N = N;
  g.N32 = N >> 5;
  g.tile = tile;
  g.s = tile * 32u + lane;
  g.lane = lane;
  g.digest = DIG && p.digest != nullptr;
  uint4 pfb = make_uint4(0, 0, 0, 0);
  {
    const uint32_t b0 = __ldg(p.bit_ptr + p.step_begin), b1e = __ldg(p.bit_ptr + p.step_begin + 1);
    if (b0 + threadIdx.x < b1e) pfb = __ldg(p.bitdesc + b0 + threadIdx.x);
  }
  for (uint32_t c = 0; c < p.n_cycles; c++) {
    const uint32_t par = (uint32_t)((p.cycle0 + c) & 1ull);
    g.cur = p.state[par];
    g.nxt = p.state[par ^ 1u];
    g.inp.bit = p.in.bit + (size_t)c * p.in_stride[CLS_BIT];
    g.inp.u8 = p.in.u8 + (size_t)c * p.in_stride[CLS_U8];
    g.inp.u16 = p.in.u16 + (size_t)c * p.in_stride[CLS_U16];
    g.inp.u32 = p.in.u32 + (size_t)c * p.in_stride[CLS_U32];
    g.out = p.out + (size_t)c * p.OW * N;
    unsigned long long dig = 0ull;
    uint32_t k = __ldg(p.uptr + p.step_begin * p.L + wl), ke = __ldg(p.uptr + p.step_begin * p.L + wl + 1);
    for (uint32_t step = p.step_begin; step < p.step_end; step++) {
      const uint32_t nstep = step + 1 < p.step_end ? step + 1 : p.step_begin;
      const uint32_t nk = __ldg(p.uptr + nstep * p.L + wl), nke = __ldg(p.uptr + nstep * p.L + wl + 1);
      // warm L1 with the next step's micro-ops (one 128-byte line per lane)
      for (uint32_t o = nk + 8u * lane; o < nke; o += 256u)
        asm volatile("prefetch.global.L1 [%0];" ::"l"(p.ustream + o));
      // ---- bit-sliced ops of this step (lane = op)
      {
        const uint32_t bb = __ldg(p.bit_ptr + step), be = __ldg(p.bit_ptr + step + 1);
        const uint32_t nbb = __ldg(p.bit_ptr + nstep), nbe = __ldg(p.bit_ptr + nstep + 1);
        const uint4 qb = pfb;
        if (nbb + threadIdx.x < nbe) pfb = __ldg(p.bitdesc + nbb + threadIdx.x);
        if (bb + threadIdx.x < be) exec_bit(sm, qb);
        for (uint32_t kk = bb + threadIdx.x + nthr; kk < be; kk += nthr) exec_bit(sm, __ldg(p.bitdesc + kk));
      }
      // ---- this warp's runs
      while (k < ke) {
        const uint4 h = __ldg(p.ustream + k);
        const uint4 *u = p.ustream + k + 1;
        const uint32_t n = h.y;
        k += 1u + n;
        switch (h.x) {
          case G_LOG + 0: h_log<1>(u, n, b1, h.z, h.w); break;
          case G_LOG + 1: h_log<2>(u, n, b2, h.z, h.w); break;
          case G_LOG + 2: h_log<4>(u, n, b4, h.z, h.w); break;
          case G_ARI + 0: h_ari<1>(u, n, b1, h.z, h.w); break;
          case G_ARI + 1: h_ari<2>(u, n, b2, h.z, h.w); break;
          case G_ARI + 2: h_ari<4>(u, n, b4, h.z, h.w); break;
          case G_UN + 0: h_un<1>(u, n, b1, h.z); break;
          case G_UN + 1: h_un<2>(u, n, b2, h.z); break;
          case G_UN + 2: h_un<4>(u, n, b4, h.z); break;
          case G_MUX + 0: h_mux<1>(u, n, b1, smem, lane); break;
          case G_MUX + 1: h_mux<2>(u, n, b2, smem, lane); break;
          case G_MUX + 2: h_mux<4>(u, n, b4, smem, lane); break;
          case G_CMP + 0: h_cmp<1>(u, n, b1, smem, lane, h.z); break;
          case G_CMP + 1: h_cmp<2>(u, n, b2, smem, lane, h.z); break;
          case G_CMP + 2: h_cmp<4>(u, n, b4, smem, lane, h.z); break;
          case G_FUN: h_fun(u, n, b4); break;
          case G_CONST: h_const(u, n, b4); break;
          case G_CONSTB: h_const(u, n, smem); break;
          case G_WADD: h_wadd(u, n, b4); break;
          case G_WCMP: h_wcmp(u, n, b4, smem, lane); break;
          case G_LD: {
            const Arena &A = h.w == 0 ? g.cur : h.w == 1 ? g.xnet : g.inp;
            h_ld(u, n, arena_ptr(A, h.z), h.z, N, tile, lane, smem);
            break;
          }
          case G_ST: {
            const Arena &A = h.w == 0 ? g.nxt : g.xnet;
            h_st<DIG>(u, n, arena_ptr(A, h.z), h.z, N, tile, lane, smem, h.w == 0 && g.digest, dig);
            break;
          }
          case G_MIX: h_mix(u, n, smem, lane, h.z); break;
          case G_GXLA: h_gx<0>(u, n, smem, lane, h.z); break;
          case G_GXUN: h_gx<1>(u, n, smem, lane, h.z); break;
          case G_GXCAT: h_gx<2>(u, n, smem, lane, 0); break;
          case G_GXMUX: h_gx<3>(u, n, smem, lane, 0); break;
          case G_GXCMP: h_gx<4>(u, n, smem, lane, h.z); break;
          default: exec_gen(u, n, g, dig); break;
        }
      }
      k = nk;
      ke = nke;
      asm volatile("cp.async.commit_group;" ::: "memory");
      switch (__ldg(p.step_wait + step)) {
        case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
        case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
        case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
        default: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
      }
      __syncthreads();
    }
    if (DIG && p.digest && dig) atomicXor(p.digest + (size_t)c * N + g.s, dig);
  }
}

}  // namespace v4

cudaError_t launch_eval_v4(const EvalParams &p, uint32_t smem_bytes, cudaStream_t st) {
  static bool attr_set[2] = {false, false};
  const int di = p.digest ? 1 : 0;
  cudaError_t e = cudaSuccess;
  if (!attr_set[di]) {   // the maximum is set once; smaller launches are fine
    e = di ? cudaFuncSetAttribute(v4::rtl_eval_v4_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448)
           : cudaFuncSetAttribute(v4::rtl_eval_v4_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
    if (e != cudaSuccess) return e;
    attr_set[di] = true;
  }
  dim3 grid(p.N_pad / 32u), block(32u * p.L);
  if (di) v4::rtl_eval_v4_kernel<true><<<grid, block, smem_bytes, st>>>(p);
  else v4::rtl_eval_v4_kernel<false><<<grid, block, smem_bytes, st>>>(p);
  return cudaGetLastError();
}

}  // namespace rtlsim
