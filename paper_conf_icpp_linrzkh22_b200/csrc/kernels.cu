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

}  // namespace rtlsim
