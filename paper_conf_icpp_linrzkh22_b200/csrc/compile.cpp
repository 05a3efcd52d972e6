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

static int arity(uint32_t opc) {
  switch (opc) {
    case RTLSIM_OP_COPY: case RTLSIM_OP_SEXT: case RTLSIM_OP_NOT: case RTLSIM_OP_NEG:
    case RTLSIM_OP_SLICE: case RTLSIM_OP_REDAND: case RTLSIM_OP_REDOR: case RTLSIM_OP_REDXOR:
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
  int32_t def_step;    // step that writes the slot
  int32_t last_use;    // last step that reads it (-1: dead)
  uint32_t slot;       // smem word offset
  bool bcast;          // constant: one copy of the words for all 32 stimuli
  uint32_t words() const { return slot_words(width, bcast); }
};

// First-fit allocator over shared-memory words.
struct SlotAlloc {
  std::map<uint32_t, uint32_t> free_;   // offset -> size
  uint32_t top = 0, peak = 0;
  explicit SlotAlloc(uint32_t base) : top(base), peak(base) {}
  uint32_t alloc(uint32_t n) {
    for (auto it = free_.begin(); it != free_.end(); ++it) {
      if (it->second >= n) {
        uint32_t off = it->first, sz = it->second;
        free_.erase(it);
        if (sz > n) free_[off + n] = sz - n;
        return off;
      }
    }
    uint32_t off = top;
    top += n;
    peak = std::max(peak, top);
    return off;
  }
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

int compile_program(const rtlsim_ir *ir, uint32_t op_lanes, uint32_t smem_limit_words, Program *P,
                    std::string *err) {
  if (!ir || !P) return fail(err, RTLSIM_E_ARG, "NULL ir");
  const uint32_t n = ir->n_signals;
  if (n == 0 || !ir->width || !ir->kind) return fail(err, RTLSIM_E_IR, "no signals");
  if ((ir->n_ops && !ir->ops) || (ir->n_regs && (!ir->reg_q || !ir->reg_d || !ir->reg_init)) ||
      (ir->n_consts && (!ir->const_sig || !ir->const_words)) || (ir->n_inputs && !ir->input_sig) ||
      (ir->n_outputs && !ir->output_sig))
    return fail(err, RTLSIM_E_ARG, "NULL array with non-zero count");
  Program &G = *P;
  G = Program();
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
    if (o.opcode > RTLSIM_OP_REDXOR) return fail(err, RTLSIM_E_IR, at + "bad opcode");
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

  // ---------------------------------------------------- partition order --
  const uint32_t NP = G.n_partitions;
  std::vector<uint32_t> porder;
  {
    std::vector<std::vector<uint32_t>> succ(NP);
    std::vector<uint32_t> indeg(NP, 0);
    std::vector<std::vector<char>> seen(NP);
    for (uint32_t i = 0; i < G.n_ops; i++) {
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
  for (uint32_t i = 0; i < G.n_ops; i++) {
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
  std::vector<std::vector<uint32_t>> reg_sinks(NP), out_sinks(NP);
  for (uint32_t r = 0; r < ir->n_regs; r++) reg_sinks[owner_of_sig(G.reg_d[r])].push_back(r);
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
    for (uint32_t i = 0; i < G.n_ops; i++) {
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++) used[src[k]] = 1;
    }
    for (uint32_t r = 0; r < ir->n_regs; r++) used[G.reg_d[r]] = 1;
    for (uint32_t o = 0; o < ir->n_outputs; o++) used[G.output_sig[o]] = 1;
    for (uint32_t i = 0; i < G.n_ops; i++) {
      uint32_t d = G.ops[i].dst;
      if (!used[d]) dump_words = std::max(dump_words, slot_words(G.width[d], false));
    }
  }

  struct StepDesc {
    Desc d;
    uint32_t cost;
  };
  std::vector<std::vector<StepDesc>> all_steps;   // global step list
  uint32_t peak = dump_words;
  G.part_steps.push_back(0);
  double bytes_state = 0, bytes_part = 0;

  std::vector<int32_t> vid_of(n, -1);   // per partition: signal -> value id (reset per partition)
  for (uint32_t p : porder) {
    const std::vector<uint32_t> &ops_p = part_ops[p];
    std::vector<Value> vals;
    std::vector<uint32_t> touched;
    auto vid = [&](uint32_t s) -> int32_t { return vid_of[s]; };
    auto new_val = [&](uint32_t s, uint32_t w, int32_t def_step) -> int32_t {
      vals.push_back(Value{s, w, def_step, -1, 0, false});
      return (int32_t)vals.size() - 1;
    };
    // 1. levels of the partition's own ops
    std::vector<int32_t> step_of_op;   // parallel to ops_p
    step_of_op.reserve(ops_p.size());
    std::unordered_map<uint32_t, int32_t> op_step;   // op index -> step
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
    // the partition (register D, output, cross-partition net) or is dead
    // keeps its earliest step so its operand cone is not dragged late.
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
      // second pass, forward: ops without local consumers run right after
      // their latest local operand; those with only external operands are
      // spread round-robin over the partition's steps (no bunching at step 1)
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
    for (uint32_t i : ops_p) {
      int32_t v = new_val(G.ops[i].dst, G.width[G.ops[i].dst], op_step[i]);
      vid_of[G.ops[i].dst] = v;
      touched.push_back(G.ops[i].dst);
    }
    // 2. external operands (registers, inputs, constants, other partitions'
    //    nets): loaded into a slot one step before use. Uses further apart
    //    than `reload_gap` steps get separate loads (a reload hits L1/L2) so
    //    the value does not occupy shared memory in between.
    auto is_local = [&](uint32_t s) { return G.kind[s] == RTLSIM_COMB && G.ops[def[s]].part == p; };
    std::unordered_map<uint32_t, std::vector<int32_t>> ext_uses;   // signal -> op use steps
    for (uint32_t i : ops_p) {
      const rtlsim_op &o = G.ops[i];
      uint32_t src[3] = {o.a, o.b, o.c};
      for (int k = 0; k < arity(o.opcode); k++)
        if (!is_local(src[k])) ext_uses[src[k]].push_back(op_step[i]);
    }
    // sinks: register next state, outputs, cross-partition nets; width
    // conversions (w_d != w_q) are synthesized COPY ops
    struct Sink {
      uint16_t op;       // OP_ST_REG / OP_ST_OUT / OP_ST_X
      uint32_t src_sig;  // signal whose value is stored
      int32_t src_val;   // value id (after conversion), -2-k: synthesized copy k
      uint32_t idx;      // register or output index, or xnet signal
    };
    std::vector<Sink> sinks;
    struct Synth {
      uint32_t src_sig, w;
      int32_t val, step;
    };
    std::vector<Synth> synth;
    for (uint32_t r : reg_sinks[p]) {
      uint32_t d = G.reg_d[r], wq = G.width[G.reg_q[r]];
      sinks.push_back(Sink{OP_ST_REG, d, -1, r});
      if (G.width[d] != wq) {
        synth.push_back(Synth{d, wq, -1, is_local(d) ? op_step[def[d]] + 1 : -1});
        sinks.back().src_val = -2 - (int32_t)(synth.size() - 1);
      }
      if (!is_local(d)) ext_uses[d];   // ensure a load exists
    }
    for (uint32_t o : out_sinks[p]) {
      uint32_t s = G.output_sig[o];
      sinks.push_back(Sink{OP_ST_OUT, s, -1, o});
      if (!is_local(s)) ext_uses[s];
    }
    for (uint32_t i : ops_p)
      if (is_xnet[G.ops[i].dst]) sinks.push_back(Sink{OP_ST_X, G.ops[i].dst, -1, G.ops[i].dst});
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
        for (Group &g : gs) {
          g.val = new_val(s, G.width[s], g.first - 1);
          vals[g.val].last_use = g.last;
          vals[g.val].bcast = G.kind[s] == RTLSIM_CONST && G.width[s] > 1;
          loads.push_back(Load{s, g.val, g.first - 1, &g == &gs.front()});
        }
        groups[s] = std::move(gs);
        touched.push_back(s);
      }
    }
    // value holding signal s at step st (local comb or the covering load)
    auto val_at = [&](uint32_t s, int32_t st) -> int32_t {
      if (is_local(s)) return vid(s);
      const std::vector<Group> &gs = groups.at(s);
      for (const Group &g : gs)
        if (st >= g.first - 1 && st <= g.last) return g.val;
      return gs.front().val;
    };
    // flexible consumers of an external value (sinks, conversion copies) read
    // the first load group, one step after the load
    for (auto &sy : synth) {
      int32_t src = is_local(sy.src_sig) ? vid(sy.src_sig) : groups.at(sy.src_sig).front().val;
      if (sy.step < 0) sy.step = vals[src].def_step + 1;
      sy.val = new_val(sy.src_sig, sy.w, sy.step);
      vals[src].last_use = std::max(vals[src].last_use, sy.step);
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
      }
    }
    // 4. sink steps: one after the stored value is written
    std::vector<int32_t> sink_step(sinks.size());
    for (size_t k = 0; k < sinks.size(); k++) {
      Sink &sk = sinks[k];
      int32_t v = sk.src_val <= -2 ? synth[-2 - sk.src_val].val
                  : (is_local(sk.src_sig) ? vid(sk.src_sig) : groups.at(sk.src_sig).front().val);
      sk.src_val = v;
      sink_step[k] = vals[v].def_step + 1;
      vals[v].last_use = std::max(vals[v].last_use, sink_step[k]);
    }
    // 5. number of steps
    int32_t nsteps = 0;
    for (auto &v : vals) nsteps = std::max(nsteps, std::max(v.def_step, v.last_use) + 1);
    // 6. slot allocation by liveness (dead values go to the dump region)
    {
      std::vector<std::vector<int32_t>> born(nsteps), dies(nsteps);
      for (size_t v = 0; v < vals.size(); v++) {
        if (vals[v].last_use < 0) {
          vals[v].slot = 0;   // dump
          continue;
        }
        born[vals[v].def_step].push_back((int32_t)v);
        dies[vals[v].last_use].push_back((int32_t)v);
      }
      SlotAlloc sa(dump_words);
      if (getenv("RTLSIM_DEBUG_LIVE")) {
        // live words per step by kind: reg/input/const/xnet loads vs comb values
        std::vector<std::array<double, 6>> live(nsteps);
        for (auto &v : vals) {
          if (v.last_use < 0) continue;
          int kd = v.def_step == 0 && false ? 0 : (G.kind[v.sig] == RTLSIM_COMB ? (is_local(v.sig) ? 4 : 3) : G.kind[v.sig]);
          for (int32_t t = v.def_step; t <= v.last_use; t++) live[t][kd] += v.words();
        }
        int32_t best = 0;
        double bw = 0;
        for (int32_t t = 0; t < nsteps; t++) {
          double tot = 0;
          for (double x : live[t]) tot += x;
          if (tot > bw) { bw = tot; best = t; }
        }
        fprintf(stderr, "part %u steps %d peak step %d words %.0f: in %.0f reg %.0f comb_local %.0f xnet %.0f const %.0f\n",
                p, nsteps, best, bw, live[best][RTLSIM_INPUT], live[best][RTLSIM_REG], live[best][4], live[best][3],
                live[best][RTLSIM_CONST]);
      }
      for (int32_t s = 0; s < nsteps; s++) {
        // largest first keeps wide values contiguous and packs better
        std::sort(born[s].begin(), born[s].end(),
                  [&](int32_t x, int32_t y) { return vals[x].words() > vals[y].words(); });
        for (int32_t v : born[s]) vals[v].slot = sa.alloc(vals[v].words());
        for (int32_t v : dies[s]) sa.release(vals[v].slot, vals[v].words());
      }
      peak = std::max(peak, sa.peak);
    }
    // 7. descriptors per step
    std::vector<std::vector<StepDesc>> steps(nsteps);
    // operand address: broadcast (constant) slots carry kConstSlot
    auto operand = [&](int32_t v) -> uint32_t { return vals[v].slot | (vals[v].bcast ? kConstSlot : 0u); };
    for (const Load &ld : loads) {
      uint32_t s = ld.sig, w = G.width[s];
      Desc d{};
      d.wd = (uint16_t)w;
      d.d = vals[ld.val].slot;   // LD_CONST writes the broadcast layout
      uint32_t op;
      if (G.kind[s] == RTLSIM_REG) {
        const RegInfo &ri = G.regs[reg_of[s]];
        op = OP_LD_REG; d.a = ri.row;
        if (ld.first) bytes_state += lane_bytes(w);
      } else if (G.kind[s] == RTLSIM_INPUT) {
        op = OP_LD_IN; d.a = input_row[s];
        if (ld.first) bytes_state += lane_bytes(w);
      } else if (G.kind[s] == RTLSIM_CONST) {
        op = OP_LD_CONST; d.a = (uint32_t)const_of[s];
      } else {
        op = OP_LD_X; d.a = xrow.at(s);
        if (ld.first) {
          bytes_state += lane_bytes(w);
          bytes_part += lane_bytes(w);
        }
      }
      d.w0 = op | ((uint32_t)width_class(w) << 17);
      steps[ld.step].push_back(StepDesc{d, nwords(w)});
    }
    // compute descriptor: widths, slot offsets, layout codes and flags
    auto compute_desc = [&](uint32_t opc, uint32_t wd, int32_t vd, int ar, const int32_t *src,
                            uint32_t imm) -> Desc {
      Desc d{};
      d.wd = (uint16_t)wd;
      d.d = vals[vd].slot;
      uint32_t w0 = opc | (layout_code(wd, false) << 17);
      bool wide = wd > 32;
      const uint32_t sh[3] = {8, 11, 14};
      uint16_t *ws[3] = {&d.wa, &d.wb, &d.wc};
      uint32_t *os[3] = {&d.a, &d.b, &d.c};
      for (int k = 0; k < ar; k++) {
        const Value &v = vals[src[k]];
        *ws[k] = (uint16_t)v.width;
        *os[k] = operand(src[k]);
        w0 |= layout_code(v.width, v.bcast) << sh[k];
        wide = wide || v.width > 32;
      }
      if (ar >= 2) w0 |= DF_HAS_B;
      if (ar >= 3) w0 |= DF_HAS_C;
      if (wide) w0 |= DF_WIDE;
      d.w0 = w0;
      d.aux = imm;
      return d;
    };
    for (size_t j = 0; j < ops_p.size(); j++) {
      const uint32_t i = ops_p[j];
      const rtlsim_op &o = G.ops[i];
      const int ar = arity(o.opcode);
      Desc d = compute_desc(o.opcode, G.width[o.dst], vid(o.dst), ar, op_vals[j].data(),
                            o.opcode == RTLSIM_OP_SLICE ? o.imm : 0u);
      uint32_t wmax = std::max<uint32_t>(d.wd, std::max<uint32_t>(d.wa, d.wb));
      uint32_t cost = nwords(wmax);
      G.word_ops += cost;
      if (o.opcode == RTLSIM_OP_MUL || o.opcode == RTLSIM_OP_DIVU || o.opcode == RTLSIM_OP_MODU) cost += 4;
      if (d.w0 & DF_WIDE) cost += 2;
      steps[op_step[i]].push_back(StepDesc{d, cost});
    }
    for (const Synth &sy : synth) {
      const int32_t src = is_local(sy.src_sig) ? vid(sy.src_sig) : groups.at(sy.src_sig).front().val;
      Desc d = compute_desc(RTLSIM_OP_COPY, sy.w, sy.val, 1, &src, 0u);
      steps[sy.step].push_back(StepDesc{d, nwords(std::max(sy.w, (uint32_t)d.wa))});
    }
    for (size_t k = 0; k < sinks.size(); k++) {
      const Sink &sk = sinks[k];
      Desc d{};
      d.a = operand(sk.src_val);
      uint32_t op = sk.op;
      if (sk.op == OP_ST_REG) {
        const RegInfo &ri = G.regs[sk.idx];
        d.wd = (uint16_t)ri.width; d.d = ri.row; d.aux = ri.word;
        bytes_state += lane_bytes(ri.width);
      } else if (sk.op == OP_ST_OUT) {
        d.wd = G.width[G.output_sig[sk.idx]]; d.d = out_word[sk.idx];
        bytes_state += 4.0 * nwords(d.wd);
      } else {
        d.wd = G.width[sk.idx]; d.d = xrow.at(sk.idx);
        bytes_state += lane_bytes(d.wd);
        bytes_part += lane_bytes(d.wd);
      }
      d.w0 = op | ((uint32_t)width_class(d.wd) << 17);
      steps[sink_step[k]].push_back(StepDesc{d, nwords(d.wd)});
    }
    for (auto &st : steps)
      if (!st.empty()) all_steps.push_back(std::move(st));
    G.part_steps.push_back((uint32_t)all_steps.size());
    for (uint32_t s : touched) vid_of[s] = -1;
  }

  // -------------------------------------------------------- op lanes --
  size_t total = 0;
  for (auto &st : all_steps) total += st.size();
  uint32_t L = op_lanes;
  if (L == 0) {
    double avg = all_steps.empty() ? 1.0 : (double)total / (double)all_steps.size();
    L = (uint32_t)std::max(1.0, std::min(16.0, avg / 8.0));
  }
  L = std::max<uint32_t>(1, std::min<uint32_t>(32, L));
  G.L = L;
  G.n_steps = (uint32_t)all_steps.size();
  G.step_ptr.reserve((size_t)G.n_steps * (L + 1));
  G.desc.reserve(total);
  for (auto &st : all_steps) {
    // longest-processing-time-first onto the least loaded lane
    std::stable_sort(st.begin(), st.end(), [](const StepDesc &x, const StepDesc &y) { return x.cost > y.cost; });
    std::vector<std::vector<Desc>> lanes(L);
    std::vector<uint64_t> load(L, 0);
    for (auto &sd : st) {
      uint32_t best = (uint32_t)(std::min_element(load.begin(), load.end()) - load.begin());
      lanes[best].push_back(sd.d);
      load[best] += sd.cost;
    }
    for (uint32_t l = 0; l < L; l++) {
      G.step_ptr.push_back((uint32_t)G.desc.size());
      std::stable_sort(lanes[l].begin(), lanes[l].end(),
                       [](const Desc &x, const Desc &y) { return (x.w0 & 0xFFu) < (y.w0 & 0xFFu); });
      G.desc.insert(G.desc.end(), lanes[l].begin(), lanes[l].end());
    }
  }
  G.step_ptr.push_back((uint32_t)G.desc.size());
  G.smem_words = std::max<uint32_t>(peak, 1);
  if (smem_limit_words && G.smem_words > smem_limit_words)
    return fail(err, RTLSIM_E_NOMEM,
                "per-tile working set of " + std::to_string(G.smem_words * 4) +
                    " bytes exceeds the shared-memory limit of " + std::to_string(smem_limit_words * 4));

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

}  // namespace rtlsim
