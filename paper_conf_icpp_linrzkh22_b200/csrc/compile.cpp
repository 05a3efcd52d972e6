// compile.cpp — IR validation, levelization, partition schedule, state layout
// and shared-memory slot allocation (host only; no CUDA).
//
// PAPER.md mapping:
//   * validation / levelization: the RTL graph must be a DAG per
//     cycle (full-cycle simulation evaluates every node once);
//   * partition DAG: macro tasks become GPU tasks with dependencies
//     (P:L269-272); partitions run in a topological order;
//   * layout: incremental width-class allocation and
//     N*offset+tid index mapping, re-derived for B200: bit-packed
//     1-bit rows, u8 / u16 / u32 rows, wide values as 32-bit word rows;
//   * per-partition steps: ops of one level are independent and run
//     concurrently on the op-lanes of a CTA (structure-level parallelism,
//     P:L159-162) while the 32 lanes of each warp are 32 stimuli
//     (stimulus-level parallelism).
#include <algorithm>
#include <array>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <numeric>
#include <queue>
#include <unordered_map>

#include "program.h"

namespace rtlsim {

// external values whose uses are more than this many steps apart are reloaded
constexpr int32_t kReloadGap = 3;
// uses of a spilled value closer than this to its definition read the slot
// (a reload must follow the spill store's step barrier and the load-ahead)
constexpr int32_t kSpillNear = 4;
// loads are issued this many steps before their first use (cp.async groups,
// awaited with a per-step wait depth just before the step barrier)
static int32_t load_ahead() {
  static const int32_t d = getenv("RTLSIM_LOAD_AHEAD") ? atoi(getenv("RTLSIM_LOAD_AHEAD")) : 2;
  return std::max(1, std::min(d, 8));
}

static int arity(uint32_t opc) {
  switch (opc) {
    case RTLSIM_OP_COPY: case RTLSIM_OP_SEXT: case RTLSIM_OP_NOT: case RTLSIM_OP_NEG:
    case RTLSIM_OP_SLICE: case RTLSIM_OP_REDAND: case RTLSIM_OP_REDOR: case RTLSIM_OP_REDXOR:
    case RTLSIM_OP_MEMRD:
      return 1;
    case RTLSIM_OP_MUX:
      return 3;
    default:
      return 2;
  }
}

static int fail(std::string *err, int code, const std::string &msg) {
  if (err) *err = msg;
  return code;
}

namespace {

struct Value {
  uint32_t sig;        // IR signal (or the register's q for synthesized copies)
  uint32_t width;
  int32_t def_step;    // step that writes the slot (-1: immediate)
  int32_t last_use;    // last step that reads it (-1: dead)
  int32_t first_use;   // first step that reads it (loads: completion deadline)
  uint32_t slot;       // smem word offset (the value itself for LC_IMM)
  uint32_t layout;     // LC_*
  uint32_t words() const { return slot_words(layout, width); }
};

// First-fit allocator over shared-memory words.
struct SlotAlloc {
  std::map<uint32_t, uint32_t> free_;   // offset -> size
  uint32_t top = 0, peak = 0;
  bool align4 = true;
  explicit SlotAlloc(uint32_t base, bool a4 = true) : top(base), peak(base), align4(a4) {}
  // slots of 4+ words start on a 16-byte boundary (16-byte cp.async row
  // copies, program.h uop loads / stores); TMEM columns need no alignment
  uint32_t alloc(uint32_t n) {
    const uint32_t al = (n >= 4 && align4) ? 4u : 1u;
    for (auto it = free_.begin(); it != free_.end(); ++it) {
      const uint32_t off = it->first, sz = it->second;
      const uint32_t a = (off + al - 1) & ~(al - 1);
      if (a + n <= off + sz) {
        free_.erase(it);
        if (a > off) free_[off] = a - off;
        if (a + n < off + sz) free_[a + n] = off + sz - a - n;
        return a;
      }
    }
    const uint32_t a = (top + al - 1) & ~(al - 1);
    if (a > top) release_raw(top, a - top);
    top = a + n;
    peak = std::max(peak, top);
    return a;
  }
  void release_raw(uint32_t off, uint32_t n) { free_[off] = n; }
  void release(uint32_t off, uint32_t n) {
    auto it = free_.emplace(off, n).first;
    // merge with next
    auto nx = std::next(it);
    if (nx != free_.end() && it->first + it->second == nx->first) {
      it->second += nx->second;
      free_.erase(nx);
    }
    // merge with previous
    if (it != free_.begin()) {
      auto pv = std::prev(it);
      if (pv->first + pv->second == it->first) {
        pv->second += it->second;
        free_.erase(it);
        it = pv;
      }
    }
    // shrink the top
    if (it->first + it->second == top) {
      top = it->first;
      free_.erase(it);
    }
  }
};

}  // namespace

// Specialized interpreter handler for a narrow op (kernels.cu fast_narrow), or
// 0 for the generic path: handler = 1 + 3 * kind + {U32, U16, U8}.
static uint32_t fast_handler(uint32_t opc, int ar, const uint32_t *lay, uint32_t ld, const uint32_t *ws,
                             uint32_t wd) {
  auto xi = [](uint32_t l) -> int { return l == LC_U32 ? 0 : l == LC_U16 ? 1 : l == LC_U8 ? 2 : -1; };
  const int X = xi(ld);
  switch (opc) {
    case RTLSIM_OP_AND: case RTLSIM_OP_OR: case RTLSIM_OP_XOR: case RTLSIM_OP_ADD: case RTLSIM_OP_SUB:
    case RTLSIM_OP_MUL:
      if (X < 0 || lay[0] != ld) return 0;
      if (lay[1] == ld) return 1 + X;                 // binary X,X->X
      if (lay[1] == LC_IMM) return 4 + X;             // binary X,IMM->X
      return 0;
    case RTLSIM_OP_COPY: case RTLSIM_OP_NOT: case RTLSIM_OP_NEG: case RTLSIM_OP_SLICE:
      return (X >= 0 && lay[0] == ld) ? 7 + X : 0;    // unary X->X
    case RTLSIM_OP_SEXT:
      return (X >= 0 && lay[0] == ld && ws[0] <= 32) ? 7 + X : 0;
    case RTLSIM_OP_MUX:   // then/else as wide as the result: no extension needed
      return (X >= 0 && lay[0] == LC_BIT && lay[1] == ld && lay[2] == ld && ws[1] <= wd && ws[2] <= wd) ? 10 + X : 0;
    case RTLSIM_OP_EQ: case RTLSIM_OP_NE: case RTLSIM_OP_LTU: case RTLSIM_OP_LEU: case RTLSIM_OP_GTU:
    case RTLSIM_OP_GEU: {
      const int A = xi(lay[0]);
      return (ld == LC_BIT && A >= 0 && lay[1] == lay[0] && ar == 2) ? 13 + A : 0;
    }
    default:
      return 0;
  }
}

int compile_program(const rtlsim_ir *ir, uint32_t op_lanes, uint32_t smem_limit_words, Program *P,
                    std::string *err, bool dce, bool fold_conv, uint32_t tmem_cols) {
  if (!ir || !P) return fail(err, RTLSIM_E_ARG, "NULL ir");
  tmem_cols = std::min<uint32_t>(tmem_cols, 512u);
  const uint32_t n = ir->n_signals;
  if (n == 0 || !ir->width || !ir->kind) return fail(err, RTLSIM_E_IR, "no signals");
  if ((ir->n_ops && !ir->ops) || (ir->n_regs && (!ir->reg_q || !ir->reg_d || !ir->reg_init)) ||
      (ir->n_consts && (!ir->const_sig || !ir->const_words)) || (ir->n_inputs && !ir->input_sig) ||
      (ir->n_outputs && !ir->output_sig))
    return fail(err, RTLSIM_E_ARG, "NULL array with non-zero count");
  Program &G = *P;
  G = Program();
  // JIT schedules balance op-lanes by generated SASS (RTLSIM_OLD_COST: the
  // interpreter's costs, for A/B)
  const bool jcost = fold_conv && !getenv("RTLSIM_OLD_COST");
  G.n_signals = n;
  G.n_ops = ir->n_ops;
  G.n_partitions = std::max<uint32_t>(1, ir->n_partitions);
  G.width.assign(ir->width, ir->width + n);
  G.kind.assign(ir->kind, ir->kind + n);
  G.ops.assign(ir->ops, ir->ops + ir->n_ops);
  G.reg_q.assign(ir->reg_q, ir->reg_q + ir->n_regs);
  G.reg_d.assign(ir->reg_d, ir->reg_d + ir->n_regs);
  G.const_sig.assign(ir->const_sig, ir->const_sig + ir->n_consts);
  G.input_sig.assign(ir->input_sig, ir->input_sig + ir->n_inputs);
  G.output_sig.assign(ir->output_sig, ir->output_sig + ir->n_outputs);

  // ------------------------------------------------------------ validate --
  for (uint32_t s = 0; s < n; s++) {
    if (G.width[s] < 1 || G.width[s] > RTLSIM_MAX_WIDTH)
      return fail(err, RTLSIM_E_IR, "signal " + std::to_string(s) + ": width out of range 1..1024");
    if (G.kind[s] > RTLSIM_CONST) return fail(err, RTLSIM_E_IR, "signal " + std::to_string(s) + ": bad kind");
  }
  std::vector<int32_t> reg_of(n, -1), const_of(n, -1), input_of(n, -1), def(n, -1);
  for (uint32_t r = 0; r < ir->n_regs; r++) {
    uint32_t q = G.reg_q[r], d = G.reg_d[r];
    if (q >= n || d >= n || G.kind[q] != RTLSIM_REG || reg_of[q] != -1)
      return fail(err, RTLSIM_E_IR, "register " + std::to_string(r) + ": bad q/d");
    reg_of[q] = (int32_t)r;
    G.RW += nwords(G.width[q]);
  }
  G.reg_init.assign(ir->reg_init, ir->reg_init + G.RW);
  uint32_t cw = 0;
  for (uint32_t k = 0; k < ir->n_consts; k++) {
    uint32_t s = G.const_sig[k];
    if (s >= n || G.kind[s] != RTLSIM_CONST || const_of[s] != -1)
      return fail(err, RTLSIM_E_IR, "const " + std::to_string(k) + ": bad signal");
    const_of[s] = (int32_t)cw;
    cw += nwords(G.width[s]);
  }
  G.const_words.assign(ir->const_words, ir->const_words + cw);
  std::vector<uint32_t> input_row(n, 0);
  for (uint32_t i = 0; i < ir->n_inputs; i++) {
    uint32_t s = G.input_sig[i];
    if (s >= n || G.kind[s] != RTLSIM_INPUT || input_of[s] != -1)
      return fail(err, RTLSIM_E_IR, "input " + std::to_string(i) + ": bad signal");
    input_of[s] = (int32_t)G.IW;
    {
      // class-formatted per-cycle input rows (N2 writes them, LD_IN copies)
      const uint32_t c = width_class(G.width[s]);
      input_row[s] = G.in_rows[c];
      for (uint32_t k = 0; k < nwords(G.width[s]); k++) {
        G.in_map.push_back(c);
        G.in_map.push_back(G.in_rows[c] + (c == CLS_U32 ? k : 0));
      }
      G.in_rows[c] += (c == CLS_U32) ? nwords(G.width[s]) : 1;
    }
    for (uint32_t k = 0; k < nwords(G.width[s]); k++) {
      uint32_t bits = std::min<uint32_t>(32, G.width[s] - 32 * k);
      G.in_mask.push_back(bits == 32 ? 0xFFFFFFFFu : ((1u << bits) - 1u));
    }
    G.IW += nwords(G.width[s]);
  }
  for (uint32_t o = 0; o < ir->n_outputs; o++) {
    if (G.output_sig[o] >= n) return fail(err, RTLSIM_E_IR, "output " + std::to_string(o) + ": bad signal");
    G.OW += nwords(G.width[G.output_sig[o]]);
  }
  for (uint32_t s = 0; s < n; s++) {
    if (G.kind[s] == RTLSIM_REG && reg_of[s] < 0) return fail(err, RTLSIM_E_IR, "REG signal without register entry");
    if (G.kind[s] == RTLSIM_CONST && const_of[s] < 0) return fail(err, RTLSIM_E_IR, "CONST signal without value");
    if (G.kind[s] == RTLSIM_INPUT && input_of[s] < 0) return fail(err, RTLSIM_E_IR, "INPUT signal not in input list");
  }
  for (uint32_t i = 0; i < G.n_ops; i++) {
    const rtlsim_op &o = G.ops[i];
    const std::string at = "op " + std::to_string(i) + ": ";
    if (o.opcode > RTLSIM_OP_MEMRD) return fail(err, RTLSIM_E_IR, at + "bad opcode");
    if (o.opcode == RTLSIM_OP_MEMRD) {
      if (o.imm >= ir->n_mems || !ir->mem_width || ir->mem_width[o.imm] != G.width[o.dst] || o.a >= n)
        return fail(err, RTLSIM_E_IR, at + "MEMRD: no such memory or width differs");
      if (G.width[o.a] > 32) return fail(err, RTLSIM_E_UNSUPPORTED, at + "MEMRD address wider than 32 bits");
    }
    if (o.dst >= n || G.kind[o.dst] != RTLSIM_COMB) return fail(err, RTLSIM_E_IR, at + "dst must be a COMB signal");
    if (def[o.dst] != -1) return fail(err, RTLSIM_E_IR, at + "multiple drivers");
    def[o.dst] = (int32_t)i;
    uint32_t src[3] = {o.a, o.b, o.c};
    for (int k = 0; k < arity(o.opcode); k++)
      if (src[k] >= n) return fail(err, RTLSIM_E_IR, at + "operand out of range");
    if (o.part >= G.n_partitions) return fail(err, RTLSIM_E_IR, at + "partition out of range");
    uint32_t wd = G.width[o.dst];
    if (o.opcode == RTLSIM_OP_MUL || o.opcode == RTLSIM_OP_DIVU || o.opcode == RTLSIM_OP_MODU) {
      if (wd > 64 || G.width[o.a] > 64 || G.width[o.b] > 64)
        return fail(err, RTLSIM_E_UNSUPPORTED, at + "MUL/DIVU/MODU wider than 64 bits");
    }
    if (o.opcode == RTLSIM_OP_SLICE && (uint64_t)o.imm + wd > G.width[o.a])
      return fail(err, RTLSIM_E_IR, at + "SLICE out of range");
  }
  for (uint32_t s = 0; s < n; s++)
    if (G.kind[s] == RTLSIM_COMB && def[s] < 0) return fail(err, RTLSIM_E_IR, "undriven COMB signal " + std::to_string(s));
  // memories: arena rows [entry word][N] (u32), write-port signals stored to
  // the port arena every cycle (applied after the cycle's partitions)
  if (ir->n_mems && (!ir->mem_width || !ir->mem_depth)) return fail(err, RTLSIM_E_ARG, "NULL memory arrays");
  if (ir->n_wports && !ir->mem_wport) return fail(err, RTLSIM_E_ARG, "NULL write ports");
  for (uint32_t m = 0; m < ir->n_mems; m++) {
    const uint32_t w = ir->mem_width[m], dpt = ir->mem_depth[m];
    if (w < 1 || w > RTLSIM_MAX_WIDTH || dpt < 1) return fail(err, RTLSIM_E_IR, "memory " + std::to_string(m) + ": bad shape");
    if ((uint64_t)G.MR + (uint64_t)dpt * nwords(w) >= (1ull << 31))
      return fail(err, RTLSIM_E_UNSUPPORTED, "memories larger than 2^31 words per stimulus");
    G.mem_width.push_back((uint16_t)w);
    G.mem_depth.push_back(dpt);
    G.mem_row0.push_back(G.MR);
    G.MR += dpt * nwords(w);
  }
  G.mem_init.assign(G.MR, 0u);
  if (ir->mem_init) std::copy(ir->mem_init, ir->mem_init + G.MR, G.mem_init.begin());
  for (uint32_t m = 0; m < G.mem_width.size(); m++)   // canonical entries: bits >= width are zero
    if (G.mem_width[m] & 31u)
      for (uint32_t e = 0; e < G.mem_depth[m]; e++)
        G.mem_init[G.mem_row0[m] + e * nwords(G.mem_width[m]) + nwords(G.mem_width[m]) - 1] &=
            (1u << (G.mem_width[m] & 31u)) - 1u;
  for (uint32_t p = 0; p < ir->n_wports; p++) {
    const uint32_t *w = ir->mem_wport + 4 * p;
    if (w[0] >= ir->n_mems || w[1] >= n || w[2] >= n || w[3] >= n)
      return fail(err, RTLSIM_E_IR, "write port " + std::to_string(p) + ": bad memory or signal");
    if (G.width[w[1]] > 32) return fail(err, RTLSIM_E_UNSUPPORTED, "write port address wider than 32 bits");
    Program::WPort wp{};
    wp.mem = w[0];
    auto port_word = [&](uint32_t sig) {
      G.port_sig.push_back(sig);
      G.port_word.push_back(G.PW);
      G.PW += nwords(G.width[sig]);
      return G.port_word.back();
    };
    wp.addr_word = port_word(w[1]);
    wp.data_word = port_word(w[2]);
    wp.data_width = G.width[w[2]];
    wp.en_word = port_word(w[3]);
    wp.en_width = G.width[w[3]];
    G.wports.push_back(wp);
  }

  // ------------------------------------------------ topological op order --
  std::vector<uint32_t> topo;
  topo.reserve(G.n_ops);
  {
    std::vector<uint32_t> indeg(G.n_ops, 0);
    std::vector<std::vector<uint32_t>> users(G.n_ops);
    for (uint32_t i = 0; i < G.n_ops; i++) {
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++)
        if (G.kind[src[k]] == RTLSIM_COMB) {
          indeg[i]++;
          users[def[src[k]]].push_back(i);
        }
    }
    std::priority_queue<uint32_t, std::vector<uint32_t>, std::greater<uint32_t>> q;  // ties by op index
    for (uint32_t i = 0; i < G.n_ops; i++)
      if (!indeg[i]) q.push(i);
    while (!q.empty()) {
      uint32_t i = q.top();
      q.pop();
      topo.push_back(i);
      for (uint32_t u : users[i])
        if (--indeg[u] == 0) q.push(u);
    }
    if (topo.size() != G.n_ops) return fail(err, RTLSIM_E_COMB_LOOP, "combinational loop among ops");
  }

  // ---------------------------------------------- dead-logic elimination --
  // Full-cycle simulation evaluates every node, but the only
  // observables are the outputs and the register state: an op
  // whose value reaches no register D, no output and no live op cannot change
  // either, so it is not scheduled (the RTL front end the paper builds on,
  // Verilator, removes such logic before code generation).
  // RTLSIM_F_NO_DCE keeps it (ablation; results are identical either way).
  std::vector<char> live(G.n_ops, 1);
  if (dce) {
    std::vector<char> need(n, 0);
    for (uint32_t r = 0; r < ir->n_regs; r++) need[G.reg_d[r]] = 1;
    for (uint32_t o = 0; o < ir->n_outputs; o++) need[G.output_sig[o]] = 1;
    for (uint32_t s : G.port_sig) need[s] = 1;   // memory write ports observe their signals
    for (auto it = topo.rbegin(); it != topo.rend(); ++it) {
      const rtlsim_op &o = G.ops[*it];
      live[*it] = need[o.dst];
      if (!live[*it]) continue;
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++) need[src[k]] = 1;
    }
    topo.erase(std::remove_if(topo.begin(), topo.end(), [&](uint32_t i) { return !live[i]; }), topo.end());
  }
  G.n_live_ops = topo.size();
  for (uint32_t i = 0; i < G.n_ops; i++) {   // algorithmic word-ops of the whole design
    const rtlsim_op &o = G.ops[i];
    uint32_t wmax = G.width[o.dst];
    if (arity(o.opcode) >= 1) wmax = std::max<uint32_t>(wmax, G.width[o.a]);
    if (arity(o.opcode) >= 2) wmax = std::max<uint32_t>(wmax, G.width[o.b]);
    G.word_ops += nwords(wmax);
  }

  // ---------------------------------------------------- partition order --
  const uint32_t NP = G.n_partitions;
  std::vector<uint32_t> porder;
  {
    std::vector<std::vector<uint32_t>> succ(NP);
    std::vector<uint32_t> indeg(NP, 0);
    std::vector<std::vector<char>> seen(NP);
    for (uint32_t i = 0; i < G.n_ops; i++) {   // the IR's partition DAG, dead logic included (validation)
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++)
        if (G.kind[src[k]] == RTLSIM_COMB) {
          uint32_t p = G.ops[def[src[k]]].part, q = o.part;
          if (p != q) {
            if (seen[p].empty()) seen[p].assign(NP, 0);
            if (!seen[p][q]) {
              seen[p][q] = 1;
              succ[p].push_back(q);
              indeg[q]++;
            }
          }
        }
    }
    std::priority_queue<uint32_t, std::vector<uint32_t>, std::greater<uint32_t>> q;
    for (uint32_t p = 0; p < NP; p++)
      if (!indeg[p]) q.push(p);
    while (!q.empty()) {
      uint32_t p = q.top();
      q.pop();
      porder.push_back(p);
      for (uint32_t s : succ[p])
        if (--indeg[s] == 0) q.push(s);
    }
    if (porder.size() != NP) return fail(err, RTLSIM_E_IR, "partition DAG has a cycle");
    // the DAG in execution-order indices (a concurrent per-cycle graph waits
    // only for these)
    std::vector<uint32_t> eidx(NP);
    for (uint32_t i = 0; i < NP; i++) eidx[porder[i]] = i;
    G.part_dep.assign(NP, {});
    for (uint32_t p = 0; p < NP; p++)
      for (uint32_t s2 : succ[p]) G.part_dep[eidx[s2]].push_back(eidx[p]);
  }
  const uint32_t P_last = porder.back();

  // ------------------------------------------------ state arena layout --
  // registers: rows per class, grouped by the partition that stores them
  auto owner_of_sig = [&](uint32_t s) -> uint32_t {
    return G.kind[s] == RTLSIM_COMB ? G.ops[def[s]].part : P_last;
  };
  G.regs.resize(ir->n_regs);
  {
    std::vector<uint32_t> order(ir->n_regs);
    std::iota(order.begin(), order.end(), 0u);
    std::vector<uint32_t> prank(NP);
    for (uint32_t i = 0; i < NP; i++) prank[porder[i]] = i;
    std::stable_sort(order.begin(), order.end(), [&](uint32_t x, uint32_t y) {
      return prank[owner_of_sig(G.reg_d[x])] < prank[owner_of_sig(G.reg_d[y])];
    });
    uint32_t word = 0;
    std::vector<uint32_t> wordidx(ir->n_regs);
    for (uint32_t r = 0; r < ir->n_regs; r++) {
      wordidx[r] = word;
      word += nwords(G.width[G.reg_q[r]]);
    }
    for (uint32_t r : order) {
      uint32_t w = G.width[G.reg_q[r]];
      uint32_t c = width_class(w);
      G.regs[r] = RegInfo{G.reg_q[r], w, c, G.rows[c], wordidx[r]};
      G.rows[c] += (c == CLS_U32) ? nwords(w) : 1;
    }
  }
  G.const_pool = G.const_words;

  // cross-partition nets
  std::vector<char> is_xnet(n, 0);
  for (uint32_t i : topo) {
    const rtlsim_op &o = G.ops[i];
    uint32_t src[3] = {o.a, o.b, o.c};
    for (int k = 0; k < arity(o.opcode); k++)
      if (G.kind[src[k]] == RTLSIM_COMB && G.ops[def[src[k]]].part != o.part) is_xnet[src[k]] = 1;
  }
  std::unordered_map<uint32_t, uint32_t> xrow;   // signal -> row in its class
  for (uint32_t s = 0; s < n; s++)
    if (is_xnet[s]) {
      uint32_t c = width_class(G.width[s]);
      xrow[s] = G.xrows[c];
      G.xrows[c] += (c == CLS_U32) ? nwords(G.width[s]) : 1;
    }

  // ----------------------------------------------- per-partition schedule --
  std::vector<std::vector<uint32_t>> part_ops(NP);
  for (uint32_t i : topo) part_ops[G.ops[i].part].push_back(i);
  std::vector<std::vector<uint32_t>> reg_sinks(NP), out_sinks(NP), port_sinks(NP);
  for (uint32_t r = 0; r < ir->n_regs; r++) reg_sinks[owner_of_sig(G.reg_d[r])].push_back(r);
  for (uint32_t k = 0; k < G.port_sig.size(); k++) port_sinks[owner_of_sig(G.port_sig[k])].push_back(k);
  for (uint32_t o = 0; o < ir->n_outputs; o++) out_sinks[owner_of_sig(G.output_sig[o])].push_back(o);
  std::vector<uint32_t> out_word(ir->n_outputs);
  for (uint32_t o = 0, w = 0; o < ir->n_outputs; o++) {
    out_word[o] = w;
    w += nwords(G.width[G.output_sig[o]]);
  }

  // dead-value dump region at offset 0: sized by the largest dead value
  uint32_t dump_words = 0;
  {
    std::vector<char> used(n, 0);
    for (uint32_t i : topo) {
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++) used[src[k]] = 1;
    }
    for (uint32_t r = 0; r < ir->n_regs; r++) used[G.reg_d[r]] = 1;
    for (uint32_t o = 0; o < ir->n_outputs; o++) used[G.output_sig[o]] = 1;
    for (uint32_t s : G.port_sig) used[s] = 1;
    for (uint32_t i : topo) {
      uint32_t d = G.ops[i].dst;
      if (!used[d]) dump_words = std::max(dump_words, slot_words(value_layout(G.width[d], false), G.width[d]));
    }
  }

  struct StepLists {
    std::vector<std::pair<Desc, uint32_t>> lane;   // descriptor, cost
    std::vector<BitDesc> bits;
    uint32_t wait = 0;                             // cp.async groups allowed pending at the step end
  };
  std::vector<StepLists> all_steps;   // global step list
  uint32_t peak = dump_words;
  G.part_steps.push_back(0);
  double bytes_state = 0, bytes_part = 0, bytes_spill = 0;
  // spill rows start after the cross-partition net rows; partitions reuse them
  uint32_t xnet_rows[4], max_spill_rows[4] = {0, 0, 0, 0};
  for (int c = 0; c < 4; c++) xnet_rows[c] = G.xrows[c];
  // spill target: the limit minus the descriptor staging buffers (128 words
  // per op-lane warp; the lane count is not known yet, assume the maximum)
  // (TMEM schedules are JIT-only: no interpreter staging buffers)
  const uint32_t stage_words = tmem_cols ? 0u : (op_lanes ? std::min<uint32_t>(op_lanes, 16) : 16) * 128u;
  const uint32_t step_cap = getenv("RTLSIM_STEP_CAP") ? (uint32_t)atoi(getenv("RTLSIM_STEP_CAP")) : 0;
  const uint32_t slot_budget =
      smem_limit_words > stage_words ? smem_limit_words - stage_words : (smem_limit_words ? 1u : 0xFFFFFFFFu);

  std::vector<int32_t> vid_of(n, -1);   // per partition: signal -> value id (reset per partition)
  int32_t last_spiller = -1;
  for (uint32_t p : porder) {
    const std::vector<uint32_t> &ops_p = part_ops[p];
    std::vector<Value> vals;
    std::vector<uint32_t> touched;
    auto vid = [&](uint32_t s) -> int32_t { return vid_of[s]; };
    auto new_val = [&](uint32_t s, uint32_t w, int32_t def_step, uint32_t layout) -> int32_t {
      vals.push_back(Value{s, w, def_step, -1, 1 << 30, 0, layout});
      return (int32_t)vals.size() - 1;
    };
    // The per-tile working set is capped at the slot budget by spilling the
    // longest-lived local values to rows of the cross-partition arena
    // (stored one step after definition, reloaded before far uses): HBM
    // bandwidth is traded for occupancy (more CTAs / warps per SM).
    std::unordered_map<uint32_t, uint32_t> spilled;   // signal -> row in the xnet arena
    uint32_t spill_rows[4] = {0, 0, 0, 0};
    auto row_of_x = [&](uint32_t sg) -> uint32_t {
      auto it = spilled.find(sg);
      return it != spilled.end() ? it->second : xrow.at(sg);
    };
    std::vector<StepLists> steps;
    std::unordered_map<uint32_t, int32_t> op_step;   // op index -> step
    // width cap of the list scheduler: 0 (levels as they are) first, then
    // halved from half the partition's mean level width while the working
    // set does not fit the budget even with spilling
    uint32_t cap = step_cap;
    int cap_tries = 0, stall = 0;
    uint32_t best_peak = 0xFFFFFFFFu;
    bool give_up = false;
    const size_t wide_base = G.wide.size();
    const auto snap = std::make_tuple(G.live_word_ops, G.n_bitops, G.n_narrow, G.n_wide, G.n_ld, G.n_st, bytes_state,
                                      bytes_part, bytes_spill);
    for (int attempt = 0;; attempt++) {
      for (uint32_t s2 : touched) vid_of[s2] = -1;
      touched.clear();
      vals.clear();
      G.wide.resize(wide_base);
      std::tie(G.live_word_ops, G.n_bitops, G.n_narrow, G.n_wide, G.n_ld, G.n_st, bytes_state, bytes_part, bytes_spill) =
          snap;
      // 1. levels of the partition's own ops (ASAP)
      op_step.clear();
      op_step.reserve(ops_p.size());
      for (uint32_t i : ops_p) {
        const rtlsim_op &o = G.ops[i];
        uint32_t src[3] = {o.a, o.b, o.c};
        int32_t lv = 1;
        for (int k = 0; k < arity(o.opcode); k++) {
          uint32_t s = src[k];
          if (G.kind[s] == RTLSIM_COMB && G.ops[def[s]].part == p) lv = std::max(lv, op_step[def[s]] + 1);
        }
        op_step[i] = lv;
      }
      // Placement that keeps values short-lived (what bounds the per-tile
      // shared-memory working set): an op whose result feeds later ops of this
      // partition runs one step before its earliest consumer (ALAP, so loads
      // and producers move next to their use); an op whose result only leaves
      // the partition (register D, output, cross-partition net) or is dead runs
      // right after its latest local operand, or, with none, round-robin over
      // the partition's steps (no bunching at step 1).
      {
        std::unordered_map<uint32_t, int32_t> first_use;   // op -> earliest consumer step
        first_use.reserve(ops_p.size());
        for (auto it = ops_p.rbegin(); it != ops_p.rend(); ++it) {
          auto f = first_use.find(*it);
          if (f != first_use.end()) op_step[*it] = f->second - 1;   // else: keep ASAP
          const int32_t st = op_step[*it];
          const rtlsim_op &o = G.ops[*it];
          uint32_t src[3] = {o.a, o.b, o.c};
          for (int k = 0; k < arity(o.opcode); k++) {
            uint32_t sg = src[k];
            if (G.kind[sg] == RTLSIM_COMB && G.ops[def[sg]].part == p) {
              auto g = first_use.find((uint32_t)def[sg]);
              if (g == first_use.end()) first_use[(uint32_t)def[sg]] = st;
              else g->second = std::min(g->second, st);
            }
          }
        }
        int32_t depth = 1;
        for (uint32_t i : ops_p) depth = std::max(depth, op_step[i]);
        uint32_t rr = 0;
        for (uint32_t i : ops_p) {
          if (first_use.count(i)) continue;
          const rtlsim_op &o = G.ops[i];
          uint32_t src[3] = {o.a, o.b, o.c};
          int32_t lv = 0;
          for (int k = 0; k < arity(o.opcode); k++) {
            uint32_t sg = src[k];
            if (G.kind[sg] == RTLSIM_COMB && G.ops[def[sg]].part == p) lv = std::max(lv, op_step[def[sg]] + 1);
          }
          op_step[i] = lv > 0 ? lv : 1 + (int32_t)(rr++ % (uint32_t)depth);
        }
      }
      // Width-capped list scheduling (a working-set bound): the placement above
      // is kept as the priority, but a step takes at most step_cap ops, so the
      // wide front of a DAG is stretched over more steps and fewer values are
      // live at once.
      if (cap > 0 && ops_p.size() > cap) {
        std::unordered_map<uint32_t, uint32_t> pending;   // op -> unscheduled local producers
        std::unordered_map<uint32_t, std::vector<uint32_t>> succ;
        pending.reserve(ops_p.size());
        for (uint32_t i : ops_p) {
          const rtlsim_op &o = G.ops[i];
          uint32_t src[3] = {o.a, o.b, o.c};
          uint32_t np = 0;
          for (int k = 0; k < arity(o.opcode); k++) {
            uint32_t sg = src[k];
            if (G.kind[sg] == RTLSIM_COMB && G.ops[def[sg]].part == p) {
              // a producer feeding two operands counts twice; its successor
              // entry is added twice too, so the count still reaches zero
              np++;
              succ[(uint32_t)def[sg]].push_back(i);
            }
          }
          pending[i] = np;
        }
        using QE = std::pair<int32_t, uint32_t>;   // (priority step, op)
        std::priority_queue<QE, std::vector<QE>, std::greater<QE>> ready;
        for (uint32_t i : ops_p)
          if (pending[i] == 0) ready.push({op_step[i], i});
        std::vector<uint32_t> now;
        int32_t t = 0;
        while (!ready.empty()) {
          t++;
          now.clear();
          while (!ready.empty() && now.size() < cap) {
            now.push_back(ready.top().second);
            ready.pop();
          }
          for (uint32_t i : now) op_step[i] = t;
          for (uint32_t i : now) {
            auto it = succ.find(i);
            if (it == succ.end()) continue;
            for (uint32_t c : it->second)
              if (--pending[c] == 0) ready.push({op_step[c], c});
          }
        }
      }
      uint32_t part_peak = 0;
    for (uint32_t i : ops_p) {
      const uint32_t d = G.ops[i].dst;
      vid_of[d] = new_val(d, G.width[d], op_step[i], value_layout(G.width[d], false));
      touched.push_back(d);
    }
    auto is_local = [&](uint32_t s) { return G.kind[s] == RTLSIM_COMB && G.ops[def[s]].part == p; };
    auto is_imm = [&](uint32_t s) { return G.kind[s] == RTLSIM_CONST && G.width[s] <= 16; };
    // 2. external operands (registers, inputs, constants > 16 bits, other
    //    partitions' nets): loaded into a slot one step before use. Uses
    //    further apart than kReloadGap steps get separate loads (a reload hits
    //    L1/L2) so the value does not occupy shared memory in between.
    //    Constants <= 16 bits are immediates in the descriptors.
    std::unordered_map<uint32_t, std::vector<int32_t>> ext_uses;   // signal -> op use steps
    // spilled local values: far uses (>= def + kSpillNear) read reloads of the
    // spill row instead of keeping the slot live
    std::unordered_map<uint32_t, std::vector<int32_t>> spill_uses;   // spilled signal -> far use steps
    auto far_use = [&](uint32_t sg, int32_t st) {
      return spilled.count(sg) && is_local(sg) && st >= op_step[def[sg]] + kSpillNear;
    };
    for (uint32_t i : ops_p) {
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++) {
        if (!is_local(src[k]) && !is_imm(src[k])) ext_uses[src[k]].push_back(op_step[i]);
        else if (far_use(src[k], op_step[i])) spill_uses[src[k]].push_back(op_step[i]);
      }
    }
    // sinks: register next state, outputs, cross-partition nets. A sink
    // whose source has another width (register q <= d mod 2^w_q) or is a
    // constant reads a synthesized COPY.
    struct Sink {
      uint32_t code;     // CODE_ST_REG / CODE_ST_OUT / CODE_ST_X
      uint32_t src_sig;  // signal whose value is stored
      int32_t src_val;   // value id; -2-k: synthesized copy k
      uint32_t idx;      // register or output index, or xnet signal
      bool conv = false; // register store converting the width itself (CODE_ST_REGC)
    };
    std::vector<Sink> sinks;
    struct Synth {
      uint32_t src_sig, w;
      int32_t val, step;
    };
    std::vector<Synth> synth;
    auto add_sink = [&](uint32_t code, uint32_t s, uint32_t w_target, uint32_t idx) {
      sinks.push_back(Sink{code, s, -1, idx});
      if (fold_conv && code == CODE_ST_REG && G.kind[s] != RTLSIM_CONST && G.width[s] != w_target) {
        // JIT kernels store q <- d mod 2^w_q straight from d's slot: no
        // conversion copy, no extra slot live until the store
        sinks.back().conv = true;
      } else if (G.width[s] != w_target || G.kind[s] == RTLSIM_CONST) {
        synth.push_back(Synth{s, w_target, -1, is_local(s) ? op_step[def[s]] + 1 : -1});
        sinks.back().src_val = -2 - (int32_t)(synth.size() - 1);
      }
      if (!is_local(s) && !is_imm(s)) ext_uses[s];   // ensure a load exists
    };
    for (uint32_t r : reg_sinks[p]) add_sink(CODE_ST_REG, G.reg_d[r], G.width[G.reg_q[r]], r);
    for (uint32_t o : out_sinks[p]) add_sink(CODE_ST_OUT, G.output_sig[o], G.width[G.output_sig[o]], o);
    for (uint32_t k : port_sinks[p]) add_sink(CODE_ST_PORT, G.port_sig[k], G.width[G.port_sig[k]], k);
    for (uint32_t i : ops_p)
      if (is_xnet[G.ops[i].dst] || (spilled.count(G.ops[i].dst) && spill_uses.count(G.ops[i].dst)))
        add_sink(CODE_ST_X, G.ops[i].dst, G.width[G.ops[i].dst], G.ops[i].dst);
    // immediates: one pseudo-value per constant, always available, no slot
    std::unordered_map<uint32_t, int32_t> imm_val;
    auto imm_of = [&](uint32_t s) -> int32_t {
      auto it = imm_val.find(s);
      if (it != imm_val.end()) return it->second;
      int32_t v = new_val(s, G.width[s], -1, LC_IMM);
      vals[v].slot = G.const_words[(uint32_t)const_of[s]] & (G.width[s] == 32 ? 0xFFFFFFFFu : ((1u << G.width[s]) - 1u));
      imm_val[s] = v;
      return v;
    };
    // load groups
    struct Load {
      uint32_t sig;
      int32_t val, step;
      bool first;   // first load of the signal in this partition (HBM traffic)
    };
    std::vector<Load> loads;
    struct Group {
      int32_t first, last, val;
    };
    std::unordered_map<uint32_t, std::vector<Group>> groups;
    {
      std::vector<uint32_t> sigs;
      sigs.reserve(ext_uses.size());
      for (auto &kv : ext_uses) sigs.push_back(kv.first);
      std::sort(sigs.begin(), sigs.end());
      for (uint32_t s : sigs) {
        std::vector<int32_t> &u = ext_uses[s];
        std::sort(u.begin(), u.end());
        u.erase(std::unique(u.begin(), u.end()), u.end());
        std::vector<Group> gs;
        if (u.empty()) gs.push_back(Group{1, 1, -1});   // sink-only: load at step 0
        for (int32_t st : u) {
          if (gs.empty() || st - gs.back().last > (int32_t)kReloadGap) gs.push_back(Group{st, st, -1});
          else gs.back().last = st;
        }
        for (size_t g = 0; g < gs.size(); g++) {
          const int32_t issue = std::max(0, gs[g].first - load_ahead());
          gs[g].val = new_val(s, G.width[s], issue, value_layout(G.width[s], G.kind[s] == RTLSIM_CONST));
          vals[gs[g].val].last_use = gs[g].last;
          loads.push_back(Load{s, gs[g].val, issue, g == 0});
        }
        groups[s] = std::move(gs);
      }
      // reloads of spilled values: issued after the spill store (def + 1) is
      // visible, i.e. at step >= def + 2
      std::vector<uint32_t> ssigs;
      for (auto &kv : spill_uses) ssigs.push_back(kv.first);
      std::sort(ssigs.begin(), ssigs.end());
      for (uint32_t s : ssigs) {
        std::vector<int32_t> &u = spill_uses[s];
        std::sort(u.begin(), u.end());
        u.erase(std::unique(u.begin(), u.end()), u.end());
        const int32_t dstep = op_step[def[s]];
        std::vector<Group> gs;
        for (int32_t st : u) {
          if (gs.empty() || st - gs.back().last > (int32_t)kReloadGap) gs.push_back(Group{st, st, -1});
          else gs.back().last = st;
        }
        for (size_t g = 0; g < gs.size(); g++) {
          const int32_t issue = std::max(dstep + 2, gs[g].first - load_ahead());
          gs[g].val = new_val(s, G.width[s], issue, value_layout(G.width[s], false));
          vals[gs[g].val].last_use = gs[g].last;
          loads.push_back(Load{s, gs[g].val, issue, false});
        }
        groups[s] = std::move(gs);
      }
    }
    // value holding signal s at step st (local comb, immediate, or the covering load)
    auto val_at = [&](uint32_t s, int32_t st) -> int32_t {
      if (is_local(s) && !far_use(s, st)) return vid(s);
      if (is_imm(s)) return imm_of(s);
      const std::vector<Group> &gs = groups.at(s);
      for (const Group &g : gs)
        if (st >= g.first - 1 && st <= g.last) return g.val;
      return gs.front().val;
    };
    auto flex_src = [&](uint32_t s) -> int32_t {   // first value of s in this partition
      if (is_local(s)) return vid(s);
      if (is_imm(s)) return imm_of(s);
      return groups.at(s).front().val;
    };
    // flexible consumers of an external value (sinks, conversion copies) read
    // the first load group, one step after the load
    for (auto &sy : synth) {
      int32_t src = flex_src(sy.src_sig);
      if (sy.step < 0) sy.step = std::max(vals[src].def_step, 0) + 1;
      sy.val = new_val(sy.src_sig, sy.w, sy.step, value_layout(sy.w, false));
      vals[src].last_use = std::max(vals[src].last_use, sy.step);
      vals[src].first_use = std::min(vals[src].first_use, sy.step);
    }
    // 3. uses by ops
    std::vector<std::array<int32_t, 3>> op_vals(ops_p.size());
    for (size_t j = 0; j < ops_p.size(); j++) {
      const uint32_t i = ops_p[j];
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++) {
        int32_t v = val_at(src[k], op_step[i]);
        op_vals[j][k] = v;
        vals[v].last_use = std::max(vals[v].last_use, op_step[i]);
        vals[v].first_use = std::min(vals[v].first_use, op_step[i]);
      }
    }
    // 4. sink steps: one after the stored value is written
    std::vector<int32_t> sink_step(sinks.size());
    for (size_t k = 0; k < sinks.size(); k++) {
      Sink &sk = sinks[k];
      int32_t v = sk.src_val <= -2 ? synth[-2 - sk.src_val].val : flex_src(sk.src_sig);
      sk.src_val = v;
      sink_step[k] = std::max(vals[v].def_step, 0) + 1;
      vals[v].last_use = std::max(vals[v].last_use, sink_step[k]);
      vals[v].first_use = std::min(vals[v].first_use, sink_step[k]);
    }
    // 5. number of steps
    int32_t nsteps = 0;
    for (auto &v : vals) nsteps = std::max(nsteps, std::max(v.def_step, v.last_use) + 1);
    // 6. slot allocation by liveness (dead values go to the dump region,
    //    immediates take no slot)
    {
      std::vector<std::vector<int32_t>> born(nsteps), dies(nsteps);
      for (size_t v = 0; v < vals.size(); v++) {
        if (vals[v].layout == LC_IMM) continue;
        if (vals[v].last_use < 0) {
          vals[v].slot = 0;   // dump
          continue;
        }
        born[vals[v].def_step].push_back((int32_t)v);
        dies[vals[v].last_use].push_back((int32_t)v);
      }
      // (r2) TMEM: U32-layout values computed by this partition's ops (not
      // cp.async load targets, not operands / results of the generic wide
      // path, which addresses shared memory) take TMEM columns while they fit
      std::vector<char> tm_ok(vals.size(), 0);
      if (tmem_cols) {
        for (size_t v = 0; v < vals.size(); v++) tm_ok[v] = vals[v].layout == LC_U32 && vals[v].def_step >= 0;
        for (const Load &ld : loads) tm_ok[ld.val] = 0;
        for (size_t j = 0; j < ops_p.size(); j++) {
          const rtlsim_op &o = G.ops[ops_p[j]];
          if (o.opcode != RTLSIM_OP_SHL && o.opcode != RTLSIM_OP_SHRL && o.opcode != RTLSIM_OP_SHRA) continue;
          const int32_t vd = vid(o.dst), va = op_vals[j][0], vb = op_vals[j][1];
          if (vd < 0 || va < 0 || vb < 0) continue;
          const bool wide = vals[vd].width > 32 || vals[va].width > 32 || vals[vb].width > 32 ||
                            vals[va].layout == LC_BCAST || vals[vb].layout == LC_BCAST;
          if (wide) tm_ok[vd] = tm_ok[va] = tm_ok[vb] = 0;
        }
      }
      SlotAlloc sa((dump_words + 3u) & ~3u), ta(0);
      for (int32_t s = 0; s < nsteps; s++) {
        // largest first keeps wide values contiguous and packs better
        std::sort(born[s].begin(), born[s].end(),
                  [&](int32_t x, int32_t y) { return vals[x].words() > vals[y].words(); });
        for (int32_t v : born[s]) {
          if (tm_ok[v]) {
            const uint32_t nw = nwords(vals[v].width), col = ta.alloc(nw);
            if (col + nw <= tmem_cols) {
              vals[v].slot = kTmemBase + 32u * col;
              continue;
            }
            ta.release(col, nw);
          }
          vals[v].slot = sa.alloc(vals[v].words());
        }
        for (int32_t v : dies[s]) {
          if (in_tmem(vals[v].slot) && vals[v].layout == LC_U32)
            ta.release((vals[v].slot - kTmemBase) / 32u, nwords(vals[v].width));
          else
            sa.release(vals[v].slot, vals[v].words());
        }
      }
      part_peak = sa.peak;
      G.tmem_cols = std::max(G.tmem_cols, std::min(ta.peak, tmem_cols));
    }
      if (part_peak > slot_budget) {
        // spill more: local values live (beyond their near uses) across the
        // steps whose working set exceeds the budget, most words x over-budget
        // steps first, until the projected working set fits
        std::vector<double> live(nsteps + 1, 0.0);
        for (auto &v : vals) {
          if (v.layout == LC_IMM || v.last_use < 0 || (v.layout == LC_U32 && in_tmem(v.slot))) continue;
          for (int32_t t = v.def_step; t <= v.last_use; t++) live[t] += v.words();
        }
        // live words that fit the budget, given the allocator's fragmentation
        const double max_live = *std::max_element(live.begin(), live.end());
        const double target = 0.98 * slot_budget * std::min(1.0, max_live / std::max(1u, part_peak));
        std::vector<std::pair<double, uint32_t>> cand;
        for (auto &v : vals) {
          if (v.layout == LC_IMM || v.last_use < 0 || !is_local(v.sig) || spilled.count(v.sig)) continue;
          if (v.layout == LC_U32 && in_tmem(v.slot)) continue;   // spilling it frees no shared memory
          if (vid(v.sig) < 0 || &vals[vid(v.sig)] != &v) continue;   // the defining value only
          int32_t over = 0;
          for (int32_t t = v.def_step + kSpillNear; t <= v.last_use; t++) over += live[t] > target;
          if (over > 0) cand.push_back({(double)v.words() * over, v.sig});
        }
        if (part_peak < best_peak) {
          stall = (part_peak * 100ull > best_peak * 99ull) ? stall + 1 : 0;
          best_peak = part_peak;
        } else {
          stall++;
        }
        const bool last_try = cand.empty() || stall >= 3 || attempt >= 24;
        if (getenv("RTLSIM_SPILL_DEBUG") && (attempt == 0 || last_try) && getenv("RTLSIM_SPILL_DEBUG")[0] == '2') {
          // live words per step by category: 0 local short, 1 local long, 2 loads, 3 other
          std::vector<std::array<double, 4>> livec(nsteps + 1, {0, 0, 0, 0});
          for (auto &v : vals) {
            if (v.layout == LC_IMM || v.last_use < 0) continue;
            int cat = 3;
            if (is_local(v.sig) && vid(v.sig) >= 0 && &vals[vid(v.sig)] == &v)
              cat = v.last_use - v.def_step >= kSpillNear ? 1 : 0;
            else if (!is_local(v.sig)) cat = 2;
            for (int32_t t = v.def_step; t <= v.last_use; t++) livec[t][cat] += v.words();
          }
          int32_t best = 0;
          double bw = 0;
          for (int32_t t = 0; t < nsteps; t++) {
            double w = livec[t][0] + livec[t][1] + livec[t][2] + livec[t][3];
            if (w > bw) bw = w, best = t;
          }
          fprintf(stderr, "  nsteps %d peak step %d live %.0f: short %.0f long %.0f loads %.0f other %.0f\n", nsteps, best,
                  bw, livec[best][0], livec[best][1], livec[best][2], livec[best][3]);
        }
        if (cand.empty() || stall >= 3 || attempt >= 24) {
          // spilling stalls: narrow the schedule instead and start over
          if (cap_tries >= 4 || (cap && cap <= 16)) {
            give_up = true;   // emit as is; the limit check below reports E_NOMEM
            if (getenv("RTLSIM_SPILL_DEBUG"))
              fprintf(stderr, "part %u gives up: peak %u budget %u cap %u\n", p, part_peak, slot_budget, cap);
            goto emit;
          }
          int32_t depth = 1;
          for (uint32_t i : ops_p) depth = std::max(depth, op_step[i]);
          cap = cap ? cap / 2 : std::max<uint32_t>(16, (uint32_t)(ops_p.size() / (size_t)depth / 2));
          cap_tries++;
          if (getenv("RTLSIM_SPILL_DEBUG"))
            fprintf(stderr, "part %u: peak %u budget %u, step cap -> %u\n", p, part_peak, slot_budget, cap);
          stall = 0;
          best_peak = 0xFFFFFFFFu;
          attempt = -1;
          spilled.clear();
          for (int c = 0; c < 4; c++) spill_rows[c] = 0;
          continue;
        }
        std::sort(cand.rbegin(), cand.rend());
        std::vector<uint32_t> take;
        for (auto &cv : cand) {
          const Value &v = vals[vid(cv.second)];
          bool need = false;
          for (int32_t t = v.def_step + kSpillNear; t <= v.last_use && !need; t++) need = live[t] > target;
          if (!need) continue;
          for (int32_t t = v.def_step + kSpillNear; t <= v.last_use; t++) live[t] -= v.words();
          take.push_back(cv.second);
        }
        if (getenv("RTLSIM_SPILL_DEBUG") && getenv("RTLSIM_SPILL_DEBUG")[0] == '2')
          fprintf(stderr, "part %u attempt %d peak %u budget %u cand %zu spilled %zu\n", p, attempt, part_peak,
                  slot_budget, cand.size(), spilled.size());
        for (uint32_t sg : take) {
          if (is_xnet[sg]) {
            spilled[sg] = xrow.at(sg);   // its cross-partition row already holds it
          } else {
            const uint32_t c = width_class(G.width[sg]);
            spilled[sg] = xnet_rows[c] + spill_rows[c];
            spill_rows[c] += (c == CLS_U32) ? nwords(G.width[sg]) : 1;
          }
        }
        continue;
      }
    emit:
    // 7. descriptors per step
    steps.assign(nsteps, StepLists{});
    for (const Load &ld : loads) {
      const uint32_t s = ld.sig, w = G.width[s];
      Desc d{};
      d.y = vals[ld.val].slot;
      uint32_t code;
      if (G.kind[s] == RTLSIM_REG) {
        code = CODE_LD_REG;
        d.z = G.regs[reg_of[s]].row;
        if (ld.first) bytes_state += lane_bytes(w);
      } else if (G.kind[s] == RTLSIM_INPUT) {
        code = CODE_LD_IN;
        d.z = input_row[s];
        if (ld.first) bytes_state += lane_bytes(w);
      } else if (G.kind[s] == RTLSIM_CONST) {
        code = CODE_LD_CONST;
        d.z = (uint32_t)const_of[s];
      } else {
        code = CODE_LD_X;
        d.z = row_of_x(s);
        if (spilled.count(s) && is_local(s)) {
          bytes_state += lane_bytes(w);
          bytes_spill += lane_bytes(w);
        } else if (ld.first) {
          bytes_state += lane_bytes(w);
          bytes_part += lane_bytes(w);
        }
      }
      d.x = code | (width_class(w) << 8) | (nwords(w) << 12) | ((vals[ld.val].layout == LC_BCAST ? 1u : 0u) << 18);
      G.n_ld++;
      steps[ld.step].lane.push_back({d, jcost ? 1 + 4 * nwords(w) : 1 + nwords(w)});
    }
    // compute op -> bit-sliced, narrow or wide descriptor
    auto emit_compute = [&](uint32_t opc, int32_t vd, int ar, const int32_t *src, uint32_t imm, int32_t step) {
      const Value &D = vals[vd];
      bool allbit = D.width == 1 && opc != RTLSIM_OP_MEMRD, narrow = D.width <= 32;
      for (int k = 0; k < ar; k++) {
        const Value &v = vals[src[k]];
        allbit = allbit && v.width == 1;
        narrow = narrow && v.width <= 32 && v.layout != LC_BCAST;
      }
      uint32_t wmax = D.width;
      for (int k = 0; k < std::min(ar, 2); k++) wmax = std::max(wmax, vals[src[k]].width);
      G.live_word_ops += nwords(wmax);
      if (allbit) {
        BitDesc b{};
        uint32_t f[3] = {0, 0, 0}, immf = 0;
        for (int k = 0; k < ar; k++) {
          f[k] = vals[src[k]].slot;
          if (vals[src[k]].layout == LC_IMM) immf |= 1u << k;
        }
        // operands the op does not have are immediate zeros: no evaluator
        // reads a placeholder slot (such a read races with the slot's writer)
        for (int k = ar; k < 3; k++) immf |= 1u << k;
        b.x = bit_lut(opc) | (immf << 8);
        b.y = D.slot | (f[0] << 16);
        b.z = f[1] | (f[2] << 16);
        steps[step].bits.push_back(b);
        G.n_bitops++;
        return;
      }
      if (narrow) {
        Desc d{};
        uint32_t lay[3] = {0, 0, 0}, off[3] = {0, 0, 0}, wsrc[3] = {1, 1, 1};
        for (int k = 0; k < ar; k++) {
          lay[k] = vals[src[k]].layout;
          off[k] = vals[src[k]].slot;
          wsrc[k] = vals[src[k]].width;
        }
        d.x = opc | (lay[0] << 8) | (lay[1] << 11) | (lay[2] << 14) | (D.layout << 17) | (D.width << 20) |
              (wsrc[0] << 26);
        d.y = D.slot | (off[0] << 16);
        d.z = opc == RTLSIM_OP_MEMRD ? imm : off[1] | (off[2] << 16);   // MEMRD: the memory
        d.w = wsrc[1] | (imm << 6) | ((ar >= 2 ? 1u : 0u) << 11) | ((ar >= 3 ? 1u : 0u) << 12) |
              (fast_handler(opc, ar, lay, D.layout, wsrc, D.width) << 13);
        G.n_narrow++;
        // lane-balancing cost: interpreter issue slots, or (JIT schedules,
        // fold_conv) the SASS the generated code takes (RTLSIM_JIT_STATS)
        uint32_t cost = (opc == RTLSIM_OP_DIVU || opc == RTLSIM_OP_MODU) ? 6 : 2;
        if (jcost) cost = (opc == RTLSIM_OP_DIVU || opc == RTLSIM_OP_MODU) ? 20 : D.layout == LC_BIT ? 12 : 9;
        steps[step].lane.push_back({d, cost});
        return;
      }
      WideRec r{};
      r.op = opc;
      r.wd = (uint16_t)D.width;
      r.d = D.slot;
      uint16_t *ws[3] = {&r.wa, &r.wb, &r.wc};
      uint32_t *os[3] = {&r.a, &r.b, &r.c};
      for (int k = 0; k < ar; k++) {
        *ws[k] = (uint16_t)vals[src[k]].width;
        *os[k] = vals[src[k]].slot;
        r.lays |= vals[src[k]].layout << (8 * k);
      }
      r.imm = imm;
      Desc d{};
      d.x = CODE_WIDE;
      d.y = (uint32_t)G.wide.size();
      G.wide.push_back(r);
      G.n_wide++;
      steps[step].lane.push_back({d, jcost ? 6 + 6 * nwords(wmax) : 4 + 2 * nwords(wmax)});
    };
    for (size_t j = 0; j < ops_p.size(); j++) {
      const uint32_t i = ops_p[j];
      const rtlsim_op &o = G.ops[i];
      emit_compute(o.opcode, vid(o.dst), arity(o.opcode), op_vals[j].data(),
                   (o.opcode == RTLSIM_OP_SLICE || o.opcode == RTLSIM_OP_MEMRD) ? o.imm : 0u, op_step[i]);
    }
    for (const Synth &sy : synth) {
      const int32_t src = flex_src(sy.src_sig);
      emit_compute(RTLSIM_OP_COPY, sy.val, 1, &src, 0u, sy.step);
    }
    for (size_t k = 0; k < sinks.size(); k++) {
      const Sink &sk = sinks[k];
      const Value &v = vals[sk.src_val];
      Desc d{};
      d.y = v.slot;
      const uint32_t w = v.width;
      if (sk.code == CODE_ST_REG) {
        const RegInfo &ri = G.regs[sk.idx];
        d.z = ri.row;
        d.w = ri.word;
        bytes_state += lane_bytes(ri.width);
      } else if (sk.code == CODE_ST_OUT) {
        d.z = out_word[sk.idx];
        bytes_state += 4.0 * nwords(w);
      } else if (sk.code == CODE_ST_PORT) {
        d.z = G.port_word[sk.idx];
        bytes_state += 4.0 * nwords(w);
      } else {
        d.z = row_of_x(sk.idx);
        bytes_state += lane_bytes(w);
        if (is_xnet[sk.idx]) bytes_part += lane_bytes(w);
        else bytes_spill += lane_bytes(w);
      }
      d.x = sk.code | (width_class(w) << 8) | (nwords(w) << 12) | (v.layout << 18);
      uint32_t cost = jcost ? 5 * nwords(w) : 1 + nwords(w);
      if (sk.conv) {
        const RegInfo &ri = G.regs[sk.idx];
        if (ri.row >= (1u << 20)) return fail(err, RTLSIM_E_UNSUPPORTED, "more than 2^20 state rows in one class");
        d.x = CODE_ST_REGC | (ri.cls << 8) | (nwords(ri.width) << 12) | (v.layout << 18) | (w << 21);
        d.z = ri.row | (ri.width << 20);
        cost = jcost ? 4 + 4 * nwords(ri.width) : 1 + nwords(ri.width);
      }
      G.n_st++;
      steps[sink_step[k]].lane.push_back({d, cost});
    }
    // wait depth: at the end of step e at most w_e of the most recent
    // per-step cp.async groups may be pending; a load issued at step i and
    // first read at step f needs w_{f-1} <= f-1-i. Drain at the last step.
    {
      const uint32_t deflt = (uint32_t)load_ahead() - 1u;
      for (auto &st : steps) st.wait = deflt;
      for (const Load &ld : loads) {
        const int32_t f = vals[ld.val].first_use;
        if (f <= 0 || f >= (1 << 30)) continue;
        const int32_t e = f - 1;
        steps[e].wait = std::min<uint32_t>(steps[e].wait, (uint32_t)std::max(0, e - ld.step));
      }
      if (!steps.empty()) steps.back().wait = 0;
    }
    // empty steps are kept (their barrier / wait depth is part of the schedule)
      peak = std::max(peak, part_peak);
      break;
    }
    for (int c = 0; c < 4; c++) max_spill_rows[c] = std::max(max_spill_rows[c], spill_rows[c]);
    {
      // partitions share the spill rows: the ones that spill run one after
      // the other even in a concurrent graph
      const uint32_t ei = (uint32_t)G.part_steps.size() - 1;
      if (spill_rows[0] | spill_rows[1] | spill_rows[2] | spill_rows[3]) {
        if (last_spiller >= 0) G.part_dep[ei].push_back((uint32_t)last_spiller);
        last_spiller = (int32_t)ei;
      }
    }
    for (auto &st : steps) all_steps.push_back(std::move(st));
    G.part_steps.push_back((uint32_t)all_steps.size());
    for (uint32_t s : touched) vid_of[s] = -1;
  }

  for (int c = 0; c < 4; c++) G.xrows[c] = xnet_rows[c] + max_spill_rows[c];
  G.b_spill = bytes_spill;

  // -------------------------------------------------------- op lanes --
  size_t total = 0;
  for (auto &st : all_steps) total += st.lane.size() + st.bits.size() / 8;
  uint32_t L = op_lanes;
  if (L == 0) {
    double avg = all_steps.empty() ? 1.0 : (double)total / (double)all_steps.size();
    L = (uint32_t)std::max(1.0, std::min(16.0, avg / 8.0));
  }
  L = std::max<uint32_t>(1, std::min<uint32_t>(16, L));
  G.L = L;
  G.n_steps = (uint32_t)all_steps.size();
  G.step_ptr.reserve((size_t)G.n_steps * L + 1);
  G.desc.reserve(total);
  G.bit_ptr.reserve(G.n_steps + 1);
  // Lane affinity (JIT schedules, RTLSIM_AFFINITY != 0): an op goes to the
  // op-lane that produced its operands in the last two steps when that lane
  // is not overloaded, so the JIT forwards them in registers instead of a
  // shared-memory round trip (the consumer is in the same warp).
  const bool affinity = fold_conv && (!getenv("RTLSIM_AFFINITY") || atoi(getenv("RTLSIM_AFFINITY")) != 0);
  std::unordered_map<uint32_t, std::pair<uint32_t, int32_t>> writer;   // slot row -> (lane, step)
  auto rows_of = [&](uint32_t off, uint32_t lay, uint32_t w, std::vector<uint32_t> &out) {
    if (lay == LC_IMM || w == 0) return;
    if (lay == LC_U32)
      for (uint32_t i = 0; i < nwords(w); i++) out.push_back(off + 32 * i);
    else out.push_back(off);
  };
  auto operands = [&](const Desc &d, std::vector<uint32_t> &src, std::vector<uint32_t> &dst) {
    const uint32_t code = d.x & 0xFFu;
    if (code < 32u) {
      const uint32_t la = (d.x >> 8) & 7u, lb = (d.x >> 11) & 7u, lc = (d.x >> 14) & 7u, ld = (d.x >> 17) & 7u;
      rows_of(d.y >> 16, la, 32, src);
      if ((d.w >> 11) & 1u) rows_of(d.z & 0xFFFFu, lb, 32, src);
      if ((d.w >> 12) & 1u) rows_of(d.z >> 16, lc, 32, src);
      rows_of(d.y & 0xFFFFu, ld, 32, dst);
    } else if (code == CODE_WIDE) {
      const WideRec &w = G.wide[d.y];
      rows_of(w.a, w.lays & 0xFFu, w.wa, src);
      rows_of(w.b, (w.lays >> 8) & 0xFFu, w.wb, src);
      rows_of(w.c, (w.lays >> 16) & 0xFFu, w.wc, src);
      rows_of(w.d, w.wd <= 32 ? value_layout(w.wd, false) : LC_U32, w.wd, dst);
    } else if (code == CODE_ST_REG || code == CODE_ST_X || code == CODE_ST_OUT || code == CODE_ST_PORT) {
      const uint32_t nw = (d.x >> 12) & 63u, lay = (d.x >> 18) & 7u;
      rows_of(d.y, lay, lay == LC_U32 ? 32 * nw : 32, src);
    } else if (code == CODE_ST_REGC) {
      const uint32_t lay = (d.x >> 18) & 7u, sw = d.x >> 21;
      rows_of(d.y, lay, sw, src);
    } else if (code == CODE_LD_CONST) {
      const uint32_t nw = (d.x >> 12) & 63u;
      if (!((d.x >> 18) & 1u)) rows_of(d.y, LC_U32, 32 * nw, dst);
    }
  };
  uint32_t part_q = 0;
  std::vector<uint32_t> srcv, dstv;
  for (size_t si = 0; si < all_steps.size(); si++) {
    auto &st = all_steps[si];
    while (part_q + 1 < G.part_steps.size() && si >= G.part_steps[part_q + 1]) {
      part_q++;
      writer.clear();   // a partition kernel starts with no live registers
    }
    G.bit_ptr.push_back((uint32_t)G.bitdesc.size());
    G.bitdesc.insert(G.bitdesc.end(), st.bits.begin(), st.bits.end());
    // longest-processing-time-first onto the least loaded lane (or the
    // producer's lane, within a slack)
    std::stable_sort(st.lane.begin(), st.lane.end(),
                     [](const std::pair<Desc, uint32_t> &x, const std::pair<Desc, uint32_t> &y) {
                       return x.second > y.second;
                     });
    std::vector<std::vector<Desc>> lanes(L);
    std::vector<uint64_t> load(L, 0);
    uint64_t step_cost = 0;
    for (auto &sd : st.lane) step_cost += sd.second;
    static const uint64_t slack_div = getenv("RTLSIM_AFFINITY_SLACK") ? std::max(1, atoi(getenv("RTLSIM_AFFINITY_SLACK"))) : 6;
    const uint64_t slack = std::max<uint64_t>(8, step_cost / L / slack_div);
    std::vector<uint32_t> score(L);
    for (auto &sd : st.lane) {
      uint32_t best = (uint32_t)(std::min_element(load.begin(), load.end()) - load.begin());
      srcv.clear();
      dstv.clear();
      if (affinity && L > 1) {
        operands(sd.first, srcv, dstv);
        std::fill(score.begin(), score.end(), 0u);
        for (uint32_t r : srcv) {
          auto it = writer.find(r);
          if (it != writer.end() && (int32_t)si - it->second.second <= 2) score[it->second.first]++;
        }
        const uint64_t lim = load[best] + slack;
        uint32_t pick = best;
        for (uint32_t l = 0; l < L; l++)
          if (load[l] <= lim && (score[l] > score[pick] || (score[l] == score[pick] && load[l] < load[pick]))) pick = l;
        best = pick;
        for (uint32_t r : dstv) writer[r] = {best, (int32_t)si};
      }
      lanes[best].push_back(sd.first);
      load[best] += sd.second;
    }
    if (getenv("RTLSIM_BALANCE_DEBUG")) {
      static double sum_max = 0, sum_avg = 0;
      static uint64_t nst = 0;
      uint64_t mx = 0, tot = 0;
      for (uint32_t l = 0; l < L; l++) mx = std::max(mx, load[l]), tot += load[l];
      sum_max += (double)mx;
      sum_avg += (double)tot / L;
      if (++nst % 500 == 0 || si + 1 == all_steps.size())
        fprintf(stderr, "balance: %llu steps, sum(max lane cost) / sum(avg) = %.3f\n", (unsigned long long)nst,
                sum_max / std::max(1.0, sum_avg));
    }
    for (uint32_t l = 0; l < L; l++) {
      G.step_ptr.push_back((uint32_t)G.desc.size());
      // loads first (their latency overlaps the step's compute; they are
      // awaited once at the step barrier), then compute ops grouped by code
      // (fewer divergent dispatch paths), stores last
      auto rank = [](const Desc &d) -> uint32_t {
        const uint32_t c = d.x & 0xFFu;
        return (c >= CODE_LD_REG && c <= CODE_LD_CONST) ? c - CODE_LD_REG : 16u + c;
      };
      std::stable_sort(lanes[l].begin(), lanes[l].end(),
                       [&](const Desc &x, const Desc &y) { return rank(x) < rank(y); });
      G.desc.insert(G.desc.end(), lanes[l].begin(), lanes[l].end());
    }
  }
  G.step_ptr.push_back((uint32_t)G.desc.size());
  G.bit_ptr.push_back((uint32_t)G.bitdesc.size());
  G.step_wait.reserve(all_steps.size());
  for (auto &st : all_steps) G.step_wait.push_back(st.wait);
  G.smem_words = std::max<uint32_t>(peak, 1);
  if (smem_limit_words && G.smem_words > smem_limit_words)
    return fail(err, RTLSIM_E_NOMEM,
                "per-tile working set of " + std::to_string(G.smem_words * 4) +
                    " bytes exceeds the shared-memory limit of " + std::to_string(smem_limit_words * 4));

  if (getenv("RTLSIM_HIST")) {   // debugging aid: descriptor class histogram
    std::map<std::string, std::pair<uint64_t, uint64_t>> h;   // class -> (count, words)
    const char *ln[6] = {"U32", "BIT", "U16", "U8", "IMM", "BC"};
    for (const Desc &q : G.desc) {
      const uint32_t code = q.x & 0xFFu;
      char k[96];
      if (code < 32u) {
        const bool hb = (q.w >> 11) & 1u, hc = (q.w >> 12) & 1u;
        snprintf(k, sizeof k, "N op%02u %s,%s,%s->%s", code, ln[(q.x >> 8) & 7u], hb ? ln[(q.x >> 11) & 7u] : "-",
                 hc ? ln[(q.x >> 14) & 7u] : "-", ln[(q.x >> 17) & 7u]);
        h[k].first++;
        h[k].second++;
      } else if (code == CODE_WIDE) {
        const WideRec &r = G.wide[q.y];
        snprintf(k, sizeof k, "W op%02u", r.op);
        h[k].first++;
        h[k].second += nwords(std::max<uint32_t>(r.wd, std::max<uint32_t>(r.wa, r.wb)));
      } else {
        snprintf(k, sizeof k, "M code%u cls%u", code, (q.x >> 8) & 3u);
        h[k].first++;
        h[k].second += (q.x >> 12) & 63u;
      }
    }
    std::vector<std::pair<uint64_t, std::string>> v;
    for (auto &kv : h) v.push_back({kv.second.first, kv.first + " words " + std::to_string(kv.second.second)});
    std::sort(v.rbegin(), v.rend());
    for (size_t i = 0; i < v.size() && i < 80; i++) fprintf(stderr, "%8llu %s\n", (unsigned long long)v[i].first, v[i].second.c_str());
  }

  // ---------------------------------------------------------- stats --
  double bf = 0;
  for (uint32_t r = 0; r < ir->n_regs; r++) bf += 2.0 * lane_bytes(G.width[G.reg_q[r]]);
  for (uint32_t i = 0; i < ir->n_inputs; i++) bf += lane_bytes(G.width[G.input_sig[i]]);
  for (uint32_t o = 0; o < ir->n_outputs; o++) bf += lane_bytes(G.width[G.output_sig[o]]);
  G.b_floor = bf;
  G.b_state = bytes_state;
  G.b_part = bytes_part;
  return RTLSIM_OK;
}

// Truth table of an op on 1-bit operands / 1-bit result (DESIGN.md §3 table
// restricted to width 1): bit k = f(a = k & 1, b = (k >> 1) & 1, c = k >> 2).
uint32_t bit_lut(uint32_t opc) {
  uint32_t lut = 0;
  for (uint32_t k = 0; k < 8; k++) {
    const uint32_t a = k & 1u, b = (k >> 1) & 1u, c = (k >> 2) & 1u;
    uint32_t r = 0;
    switch (opc) {
      case RTLSIM_OP_COPY: case RTLSIM_OP_SEXT: case RTLSIM_OP_NEG: case RTLSIM_OP_SLICE:
      case RTLSIM_OP_REDAND: case RTLSIM_OP_REDOR: case RTLSIM_OP_REDXOR: case RTLSIM_OP_SHRA:
        r = a; break;                                   // SHRA: b >= 1 fills with the sign = a
      case RTLSIM_OP_NOT: r = a ^ 1u; break;
      case RTLSIM_OP_AND: case RTLSIM_OP_MUL: case RTLSIM_OP_DIVU: r = a & b; break;   // a/1 = a, a/0 = 0
      case RTLSIM_OP_OR: r = a | b; break;
      case RTLSIM_OP_XOR: case RTLSIM_OP_ADD: case RTLSIM_OP_SUB: case RTLSIM_OP_NE: r = a ^ b; break;
      case RTLSIM_OP_MODU: r = 0; break;               // a % 1 = 0, a % 0 = 0
      case RTLSIM_OP_EQ: r = (a ^ b) ^ 1u; break;
      case RTLSIM_OP_LTU: r = (a ^ 1u) & b; break;
      case RTLSIM_OP_LEU: r = (a ^ 1u) | b; break;
      case RTLSIM_OP_GTU: r = a & (b ^ 1u); break;
      case RTLSIM_OP_GEU: r = a | (b ^ 1u); break;
      case RTLSIM_OP_LTS: r = a & (b ^ 1u); break;     // 1-bit signed: 1 means -1
      case RTLSIM_OP_LES: r = a | (b ^ 1u); break;
      case RTLSIM_OP_GTS: r = (a ^ 1u) & b; break;
      case RTLSIM_OP_GES: r = (a ^ 1u) | b; break;
      case RTLSIM_OP_SHL: case RTLSIM_OP_SHRL: r = a & (b ^ 1u); break;   // shift by 1 >= width
      case RTLSIM_OP_MUX: r = a ? b : c; break;
      case RTLSIM_OP_CONCAT: r = b; break;             // ({a, b}) mod 2
      default: r = 0; break;
    }
    lut |= (r & 1u) << k;
  }
  return lut;
}

}  // namespace rtlsim
