// jit.h — specialized per-partition kernels (RTLSIM_F_JIT).
//
// The interpreter (kernels.cu) is issue-bound: decoding, dispatch and layout
// branches cost ~100 SASS instructions per op. PAPER.md's own flow transpiles
// the design into straight-line CUDA per partition; SURVEY
// §8(f) row 4 keeps that idea as the fallback "if the interpreter stalls on
// issue". Here the compiled schedule (the same steps, slots and layouts the
// interpreter walks) is translated into PTX — one kernel per partition, steps
// split into device functions so ptxas time stays linear — compiled in-process
// with nvPTXCompiler on all host cores and loaded with cudaLibraryLoadData.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "program.h"

namespace rtlsim {

// Kernel parameter block of a JIT partition kernel (one cycle per launch).
struct JitParams {
  uint64_t cur[4], nxt[4], xnet[4], in[4];   // arena bases per class (bit, u8, u16, u32)
  uint64_t out;                              // out rows of this cycle: [OW][N_pad] u32
  uint64_t digest;                           // digest row of this cycle [N_pad] u64, or 0
  uint64_t wide;                             // WideRec array (generic path)
  uint32_t N;                                // N_pad
  uint32_t tpc;                              // 32-stimulus tiles per CTA (warps of equal op-lane share code)
  uint64_t bittab;                           // this partition's bit-op batch table (uint4 per op) or 0
  uint64_t mem;                              // memory arena [MR][N_pad] u32 (MEMRD) or 0
  uint64_t port;                             // write-port arena [PW][N_pad] u32 (CODE_ST_PORT) or 0
  // cycles simulated by this launch (M1 persistent mode: single-partition
  // designs loop over a chunk's cycles inside the kernel; 1 otherwise) and
  // the per-cycle advance of the input / output / digest rows
  uint32_t nc, pad;
  uint64_t in_step[4];                       // bytes per cycle in the input arena, per class
  uint64_t out_step, dig_step;               // bytes per cycle of the output / digest rows
};
static_assert(sizeof(JitParams) == 240, "JitParams layout is read through offsetof in the PTX generator");

// Maximum tiles per CTA the kernels are compiled for (.maxntid 32 * L * kJitMaxTiles).
constexpr uint32_t kJitMaxTiles = 16;
// Tiles per CTA the kernels are compiled for by default (RTLSIM_JIT_TMAX
// overrides, up to kJitMaxTiles and 1024 threads per CTA).
uint32_t jit_default_tiles(bool compact = false);
// Bytes of shared memory per tile in a JIT CTA (16-byte aligned).
// (r2) TMEM schedules (computed U32 values in tensor memory, four tiles per
// CTA): RTLSIM_JIT_TMEM unset = auto (-1), 0 = off, 1 = whenever it fits
inline int jit_tmem_mode() {
  const char *e = getenv("RTLSIM_JIT_TMEM");
  return e ? (atoi(e) != 0 ? 1 : 0) : -1;
}
inline uint32_t jit_tile_bytes(const Program &G) { return ((G.smem_words * 4u) + 15u) & ~15u; }

// What the generator decided for one partition kernel beyond its PTX.
struct JitPartInfo {
  uint32_t tile_bytes = 0;          // shared memory per tile (compacted slots; 0 = jit_tile_bytes(G))
  std::vector<WideRec> wide;        // generic-path records with compacted slot offsets (or empty)
  std::vector<uint32_t> bittab;     // lane-parallel bit-op batches: {a, b, c, d} smem byte offsets per op
};

struct JitKernels {
  std::vector<cudaLibrary_t> libs;
  std::vector<uint32_t> tile_bytes; // per exec-order partition: shared memory per tile
  std::vector<uint32_t> wide_base;  // per partition: first record in d_wide (compacted records)
  WideRec *d_wide = nullptr;        // compacted generic-path records of all partitions (or null)
  std::vector<uint32_t> bit_base;   // per partition: first uint4 of its bit-op table in d_bittab
  uint32_t *d_bittab = nullptr;     // bit-op batch tables of all partitions (or null)
  bool compact = false;             // slot compaction (L == 1 kernels)
  std::vector<cudaKernel_t> kern;   // per exec-order partition (nullptr: empty partition)
  double gen_s = 0, compile_s = 0;
  bool o3 = false;
  uint32_t tmax = 1;                // tiles per CTA the kernels were built for
  uint32_t nspec = 0;               // N_pad the row offsets were specialised for (0: generic)
  size_t ptx_bytes = 0, cubin_bytes = 0;
  uint64_t sass_instructions = 0;   // .text of every partition kernel (each executed once per tile-cycle)
  uint32_t cache_hits = 0;          // partitions served from RTLSIM_JIT_CACHE
};

// PTX text of exec-order partition q (steps part_steps[q]..part_steps[q+1]).
// dig: include the per-(stimulus, cycle) digest code (check-mode variant).
// nspec: N_pad the code is specialised for (state-row offsets become
// immediates; the kernel traps on any other N), 0 = generic (row stride read
// from the launch parameters).
std::string jit_partition_ptx(const Program &G, uint32_t q, const std::string &rt_ptx, uint32_t tmax, bool dig,
                              uint32_t nspec, JitPartInfo *info = nullptr);
// Slot compaction (RTLSIM_JIT_COMPACT, default on for one op-lane): a tile is
// one warp, so only values read back from shared memory (the others stay in
// registers) get slots, allocated by step interval.
bool jit_compact(const Program &G);
// Generate + compile (nvPTXCompiler, all host cores) + load every partition.
// device < 0: generate and compile only (host-only contexts, CPU tests).
int jit_build(const Program &G, const std::string &rt_ptx_path, uint32_t smem_bytes, int device, JitKernels *out,
              std::string *err, bool dig, uint32_t nspec = 0);
void jit_free(JitKernels *k);

}  // namespace rtlsim
