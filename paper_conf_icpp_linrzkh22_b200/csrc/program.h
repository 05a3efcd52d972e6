// program.h — the compiled per-cycle schedule (host side, no CUDA types).
//
// rtlsim_load turns the IR into a Program: the paper's "kernel code
// transpilation" (§3.1) rebuilt as a layout compiler that
// emits an op stream for a hand-written interpreter kernel instead of CUDA
// source:
//   * width-class state arenas (the paper's var8/var16/var32/var64 arrays,
//     P:L578-621, plus bit-packed 1-bit rows and 32-bit word rows for >32-bit
//     values), signal-major / stimulus-minor (index mapping N*offset+tid,
//     P:L623-638);
//   * per partition (P:L674-685 macro tasks), a levelized list of steps; each
//     step's ops are independent and split over `L` op-lanes (warps sharing
//     one 32-stimulus tile); a CTA barrier separates steps;
//   * combinational values live in shared-memory slots assigned by liveness;
//     registers, inputs, constants and cross-partition nets are loaded into
//     slots by LD descriptors and stored by ST descriptors.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/rtlsim.h"

namespace rtlsim {

// internal opcodes beyond the IR's 0..30
enum : uint16_t {
  OP_LD_REG = 32,   // slot d <- state_cur[class][row a..] ; wd width
  OP_LD_X = 33,     // slot d <- xnet[class][row a..]
  OP_LD_IN = 34,    // slot d <- input class arena of cycle c [class imm][row a..]
  OP_LD_CONST = 35, // slot d <- const_pool[a..] (broadcast)
  OP_ST_REG = 40,   // state_next[class][row d..] <- slot a ; aux = register word index
  OP_ST_X = 41,     // xnet[class][row d..] <- slot a
  OP_ST_OUT = 42,   // out_chunk[c][word d..] <- slot a
};

// state / xnet arena classes (lane bytes b(w): 1/8, 1, 2, 4 per word)
enum : uint16_t { CLS_BIT = 0, CLS_U8 = 1, CLS_U16 = 2, CLS_U32 = 3 };

// operand slot flag: constant values are stored once per tile (broadcast)
constexpr uint32_t kConstSlot = 0x80000000u;
// external values whose uses are more than this many steps apart are reloaded
constexpr uint32_t kReloadGap = 3;

inline uint32_t nwords(uint32_t w) { return (w + 31u) / 32u; }
inline uint16_t width_class(uint32_t w) {
  return w == 1 ? CLS_BIT : w <= 8 ? CLS_U8 : w <= 16 ? CLS_U16 : CLS_U32;
}
// shared-memory words one value occupies per 32-stimulus tile: packed bits,
// byte lanes (2..8 bits), half-word lanes (9..16), word lanes (>16, one
// 32-word row per 32-bit word); constants keep one broadcast copy
inline uint32_t slot_words(uint32_t w, bool bcast) {
  if (w == 1) return 1u;
  if (bcast) return nwords(w);
  if (w <= 8) return 8u;
  if (w <= 16) return 16u;
  return 32u * nwords(w);
}
inline double lane_bytes(uint32_t w) {
  return w == 1 ? 0.125 : w <= 8 ? 1.0 : w <= 16 ? 2.0 : 4.0 * nwords(w);
}

// slot layout codes (operand / destination addressing in shared memory)
enum : uint32_t { LC_BIT = 0, LC_U8 = 1, LC_U16 = 2, LC_U32 = 3, LC_CONST = 4 };
inline uint32_t layout_code(uint32_t w, bool bcast) {
  return bcast ? LC_CONST : w == 1 ? LC_BIT : w <= 8 ? LC_U8 : w <= 16 ? LC_U16 : LC_U32;
}
// descriptor flags (word 0)
constexpr uint32_t DF_WIDE = 1u << 20;   // some width > 32: generic word-loop path
constexpr uint32_t DF_HAS_B = 1u << 21;
constexpr uint32_t DF_HAS_C = 1u << 22;

// 32-byte descriptor, read by the kernel as two uint4:
//   w0 = op | la << 8 | lb << 11 | lc << 14 | ld << 17 | flags   (compute ops)
//   w0 = op | class << 17                                          (LD / ST)
//   wd, wa, wb, wc widths; d, a, b, c slot offsets (or arena rows for LD/ST);
//   aux = SLICE lo, or the register word index of ST_REG (digest)
struct Desc {
  uint32_t w0;
  uint16_t wd, wa, wb, wc;
  uint32_t d, a, b, c;
  uint32_t aux;
};
static_assert(sizeof(Desc) == 32, "descriptor must be 32 bytes");

struct RegInfo {
  uint32_t sig, width, cls, row, word;   // row in its class arena; word = first RW index
};

struct Program {
  // ---- design copy
  uint32_t n_signals = 0, n_ops = 0, n_partitions = 0;
  std::vector<uint16_t> width;
  std::vector<uint8_t> kind;
  std::vector<rtlsim_op> ops;
  std::vector<uint32_t> reg_q, reg_d, reg_init, const_sig, const_words, input_sig, output_sig;
  uint32_t IW = 0, OW = 0, RW = 0;
  std::vector<uint32_t> in_mask;        // [IW] per stimulus word
  // ---- layout
  uint32_t rows[4] = {0, 0, 0, 0};      // state arena rows per class
  uint32_t xrows[4] = {0, 0, 0, 0};     // cross-partition net rows per class
  std::vector<RegInfo> regs;            // per register, IR order
  uint32_t in_rows[4] = {0, 0, 0, 0};   // per-cycle input rows per class
  std::vector<uint32_t> in_map;         // [IW][2]: class, row of each stimulus word
  std::vector<uint32_t> const_pool;     // words
  // ---- schedule
  uint32_t L = 1;                       // op-lanes (warps) per tile
  uint32_t n_steps = 0;
  std::vector<Desc> desc;
  std::vector<uint32_t> step_ptr;       // [n_steps * L + 1]: lane l of step s = [p[s*L+l], p[s*L+l+1])
  std::vector<uint32_t> part_steps;     // exec-order partition boundaries in steps (size P+1)
  uint32_t smem_words = 0;              // shared words per tile
  // ---- stats
  uint64_t word_ops = 0;
  double b_floor = 0, b_state = 0, b_part = 0;
};

// Returns RTLSIM_OK or a negative status with *err set.
int compile_program(const rtlsim_ir *ir, uint32_t op_lanes, uint32_t smem_limit_words,
                    Program *out, std::string *err);

}  // namespace rtlsim
