// kernels.h — launch wrappers for the sm_100a kernels (kernels.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "program.h"

namespace rtlsim {

// Arena pointers of one state buffer (or of the cross-partition net arena).
struct Arena {
  uint32_t *bit;   // [rows_bit][N_pad/32]
  uint8_t *u8;     // [rows_u8][N_pad]
  uint16_t *u16;   // [rows_u16][N_pad]
  uint32_t *u32;   // [rows_u32][N_pad]
};

// Per-cycle element strides of the input chunk's class arenas.
struct InStride {
  uint64_t s[4];
};

// Per register / input word: arena class and row (bit row / u8 row / u16 row /
// u32 row).
struct RegWord {
  uint32_t cls, row;
};

struct WideRec;

struct EvalParams {
  const uint4 *desc;          // 16-byte descriptors (program.h Desc), padded by 32
  const uint4 *bitdesc;       // bit-sliced ops (program.h BitDesc)
  const uint32_t *bit_ptr;    // [n_steps + 1]
  const uint32_t *step_wait;  // [n_steps] cp.async wait depth at the step end
  const WideRec *wide;        // generic-path records
  const uint32_t *step_ptr;   // [n_steps * L + 1]: lane l of step s = [p[sL+l], p[sL+l+1])
  uint32_t step_begin, step_end, L;
  uint32_t n_cycles;          // cycles processed by this launch
  uint64_t cycle0;            // absolute cycle of the first one (ping-pong parity)
  uint32_t N_pad, IW, OW;
  Arena state[2];             // ping-pong register state
  Arena xnet;                 // cross-partition nets
  Arena in;                   // class-formatted input rows of cycle 0 of this launch
  uint64_t in_stride[4];      // per-cycle element stride of each input class arena
  uint32_t desc_smem_off;     // word offset of the per-warp descriptor buffers
  uint32_t *out;              // [n_cycles][OW][N_pad]
  const uint32_t *consts;
  unsigned long long *digest; // [n_cycles][N_pad] (XOR-accumulated) or NULL
};

// N1: op-stream evaluator. grid = N_pad/32 tiles, block = 32*L threads.
cudaError_t launch_eval(const EvalParams &p, uint32_t smem_bytes, cudaStream_t st);
cudaError_t eval_set_smem(uint32_t smem_bytes);

// N2: stimulus chunk [N][nc][IW] (row pitch src_pitch words) -> per-cycle
// class-formatted input rows (map[k]: class and row of input word k), masked
// per word; stimuli >= N are zero.
cudaError_t launch_stim_transpose(const uint32_t *src, uint64_t src_pitch, uint32_t N, uint32_t N_pad,
                                  uint32_t nc, uint32_t IW, const uint32_t *mask, const RegWord *map,
                                  Arena dst, InStride st, cudaStream_t stream);
// N3: [nc][OW][N_pad] -> dst[N][*][OW] rows of nc*OW words at pitch dst_pitch words.
cudaError_t launch_out_transpose(const uint32_t *src, uint32_t N, uint32_t N_pad, uint32_t nc,
                                 uint32_t OW, uint32_t *dst, uint64_t dst_pitch, cudaStream_t st);
// digest [nc][N_pad] -> dst[N][*] rows of nc at pitch dst_pitch
cudaError_t launch_digest_transpose(const unsigned long long *src, uint32_t N, uint32_t N_pad,
                                    uint32_t nc, unsigned long long *dst, uint64_t dst_pitch,
                                    cudaStream_t st);

// N4: regs[N][RW] (src_stride 0 = broadcast one [RW] vector) -> arena
cudaError_t launch_regs_import(const uint32_t *src, uint64_t src_stride, const RegWord *map,
                               uint32_t RW, uint32_t N, uint32_t N_pad, Arena a, cudaStream_t st);
// arena -> regs[N][RW]
cudaError_t launch_regs_export(Arena a, const RegWord *map, uint32_t RW, uint32_t N,
                               uint32_t N_pad, uint32_t *dst, cudaStream_t st);
// N5 toggle coverage of one cycle (cov[k] |= OR_s R_c ^ R_{c+1}) and the
// per-stimulus register digest
cudaError_t launch_toggle_coverage(Arena cur, Arena nxt, const RegWord *map, uint32_t RW, uint32_t N,
                                   uint32_t N_pad, uint32_t *cov, cudaStream_t st);
// memories (JIT backend): write-port commit after each cycle, init, export
struct MemPortDev {
  uint32_t row0, depth, width, addr_word, data_word, data_width, en_word, en_width;
};
cudaError_t launch_mem_commit(uint32_t *mem, const uint32_t *port, const MemPortDev *ports, uint32_t n_ports,
                              uint32_t N, uint32_t N_pad, cudaStream_t st);
cudaError_t launch_mem_init(uint32_t *mem, const uint32_t *init, uint32_t MR, uint32_t N_pad, cudaStream_t st);
cudaError_t launch_mem_export(const uint32_t *mem, uint32_t MR, uint32_t N, uint32_t N_pad, uint32_t *dst,
                              cudaStream_t st);
cudaError_t launch_reg_digest(Arena a, const RegWord *map, uint32_t RW, uint32_t N, uint32_t N_pad,
                              unsigned long long *dig, cudaStream_t st);

}  // namespace rtlsim
