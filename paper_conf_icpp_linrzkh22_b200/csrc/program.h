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
//     slots by LD descriptors and stored by ST descriptors;
//   * ops whose operands and result are all 1 bit run bit-sliced: one lane per
//     op, 32 stimuli per packed word, as a 3-input truth table.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/rtlsim.h"

namespace rtlsim {

// state / xnet / input arena classes (lane bytes b(w): 1/8, 1, 2, 4 per word)
enum : uint32_t { CLS_BIT = 0, CLS_U8 = 1, CLS_U16 = 2, CLS_U32 = 3 };

// shared-memory slot layouts of a value (per 32-stimulus tile)
enum : uint32_t {
  LC_U32 = 0,    // one 32-word row per 32-bit word: word i of lane l at off + 32 i + l
  LC_BIT = 1,    // one packed word: bit l = stimulus lane l
  LC_U16 = 2,    // 32 half-word lanes (16 words)
  LC_U8 = 3,     // 32 byte lanes (8 words)
  LC_IMM = 4,    // constant <= 16 bits: the value itself is the operand field
  LC_BCAST = 5,  // constant > 32 bits: one broadcast copy of its words
};

// descriptor codes (x & 0xFF): 0..31 narrow compute op (the IR opcode)
enum : uint32_t {
  CODE_WIDE = 64,       // y = index of a WideRec
  CODE_LD_REG = 80,     // slot y <- state_cur[cls][row z .. + nw)
  CODE_LD_X = 81,       // slot y <- xnet[cls][row z ..]
  CODE_LD_IN = 82,      // slot y <- input arena of cycle c [cls][row z ..]
  CODE_LD_CONST = 83,   // slot y <- const pool[z .. + nw) (per-lane U32 or broadcast)
  CODE_ST_REG = 96,     // state_next[cls][row z ..] <- slot y ; w = register word index
  CODE_ST_X = 97,       // xnet[cls][row z ..] <- slot y
  CODE_ST_OUT = 98,     // out_chunk[c][word z ..] <- slot y
  CODE_ST_PORT = 100,   // JIT only: memory write-port word z <- slot y (port arena [PW][N])
  CODE_ST_REGC = 99,    // JIT only: state_next <- slot y converted from the source's
                        // width / layout (x >> 21) to the register's (z >> 20); z & 0xFFFFF = row
};

inline uint32_t nwords(uint32_t w) { return (w + 31u) / 32u; }

// (r2) TMEM-resident values (JIT, RTLSIM_JIT_TMEM): a U32-layout value computed
// by an op may live in tensor memory instead of a shared-memory slot. Its
// "slot" is kTmemBase + 32 * column (word i at column + i, one TMEM lane per
// stimulus), so the per-word key arithmetic off + 32 i stays the same.
constexpr uint32_t kTmemBase = 0x8000u;
inline bool in_tmem(uint32_t slot) { return slot >= kTmemBase && slot < kTmemBase + 32u * 512u; }
inline uint32_t width_class(uint32_t w) {
  return w == 1 ? CLS_BIT : w <= 8 ? CLS_U8 : w <= 16 ? CLS_U16 : CLS_U32;
}
inline double lane_bytes(uint32_t w) {
  return w == 1 ? 0.125 : w <= 8 ? 1.0 : w <= 16 ? 2.0 : 4.0 * nwords(w);
}
// layout of a signal's value in shared memory
inline uint32_t value_layout(uint32_t w, bool is_const) {
  if (is_const) return w <= 16 ? LC_IMM : (w <= 32 ? LC_U32 : LC_BCAST);
  return w == 1 ? LC_BIT : w <= 8 ? LC_U8 : w <= 16 ? LC_U16 : LC_U32;
}
inline uint32_t slot_words(uint32_t layout, uint32_t w) {
  switch (layout) {
    case LC_BIT: return 1u;
    case LC_U8: return 8u;
    case LC_U16: return 16u;
    case LC_IMM: return 0u;
    case LC_BCAST: return nwords(w);
    default: return 32u * nwords(w);
  }
}

// 16-byte descriptor (one uint4), see kernels.cu for the decoding:
//   narrow compute (code = IR opcode < 32, every width <= 32):
//     x = op | la << 8 | lb << 11 | lc << 14 | ld << 17 | wd << 20 | wa << 26
//     y = d | a << 16 ; z = b | c << 16 ; w = wb | imm << 6
//   CODE_WIDE: y = WideRec index
//   LD:  x = code | cls << 8 | nw << 12 | bcast << 18 ; y = slot ; z = row
//   ST:  x = code | cls << 8 | nw << 12 | src layout << 18 ; y = slot ; z = row ; w = aux
struct Desc {
  uint32_t x, y, z, w;
};
static_assert(sizeof(Desc) == 16, "descriptor must be 16 bytes");

// bit-sliced op (every operand and the result 1 bit): one lane evaluates a
// 3-input truth table on packed words.  x = lut | imm_a << 8 | imm_b << 9 |
// imm_c << 10 ; y = d | a << 16 ; z = b | c << 16 (an immediate operand field
// holds the constant 0 / 1)
struct BitDesc {
  uint32_t x, y, z, w;
};
static_assert(sizeof(BitDesc) == 16, "bit descriptor must be 16 bytes");

// generic (any width) op record for the out-of-line wide path; three uint4:
// {op, wd | wa << 16, wb | wc << 16, imm} {d, a, b, c} {la | lb << 8 | lc << 16, -, -, -}
struct WideRec {
  uint32_t op;
  uint16_t wd, wa, wb, wc;
  uint32_t imm;           // SLICE lo
  uint32_t d, a, b, c;    // slot offsets (or immediate values for LC_IMM)
  uint32_t lays;
  uint32_t pad[3];
};
static_assert(sizeof(WideRec) == 48, "wide record layout");

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
  std::vector<Desc> desc;               // lane lists, step-major
  std::vector<uint32_t> step_ptr;       // [n_steps * L + 1]: lane l of step s = [p[s*L+l], p[s*L+l+1])
  std::vector<BitDesc> bitdesc;         // bit-sliced ops, step-major
  std::vector<uint32_t> bit_ptr;        // [n_steps + 1]
  std::vector<uint32_t> step_wait;      // [n_steps] cp.async groups allowed pending at the step end
  std::vector<WideRec> wide;            // records referenced by CODE_WIDE
  std::vector<uint32_t> part_steps;     // exec-order partition boundaries in steps (size P+1)
  std::vector<std::vector<uint32_t>> part_dep;   // exec-order partitions each one waits for in a cycle
  uint32_t smem_words = 0;              // shared words per tile (slots)
  uint32_t tmem_cols = 0;               // (r2) TMEM columns per tile (0: no TMEM values)
  // ---- memories (ARRSEL, reading 12; JIT backend only)
  std::vector<uint16_t> mem_width;
  std::vector<uint32_t> mem_depth, mem_row0;  // first u32 row of each memory in the memory arena
  std::vector<uint32_t> mem_init;             // MR words: row r's initial value (all stimuli)
  uint32_t MR = 0;                            // memory arena rows (u32, [MR][N]) = words per stimulus
  struct WPort {
    uint32_t mem, addr_word, data_word, data_width, en_word, en_width;   // words in the port arena
  };
  std::vector<WPort> wports;                  // in port order (a later port wins)
  std::vector<uint32_t> port_sig;             // signals stored to the port arena each cycle
  std::vector<uint32_t> port_word;            // their first word
  uint32_t PW = 0;                            // port arena words per stimulus
  // ---- stats
  uint64_t word_ops = 0, n_bitops = 0, n_wide = 0, n_narrow = 0, n_ld = 0, n_st = 0;
  double b_floor = 0, b_state = 0, b_part = 0, b_spill = 0;
  uint64_t n_live_ops = 0, live_word_ops = 0;
};

// Returns RTLSIM_OK or a negative status with *err set.
int compile_program(const rtlsim_ir *ir, uint32_t op_lanes, uint32_t smem_limit_words, Program *out,
                    std::string *err, bool dce = true, bool fold_conv = false, uint32_t tmem_cols = 0);

// 3-input truth table (bit k = f(a = k&1, b = k>>1&1, c = k>>2&1)) of an IR
// opcode on 1-bit operands and a 1-bit result.
uint32_t bit_lut(uint32_t opcode);

}  // namespace rtlsim
