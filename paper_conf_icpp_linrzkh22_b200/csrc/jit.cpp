// jit.cpp — PTX generation for specialized partition kernels, in-process
// compilation with nvPTXCompiler, loading with the CUDA runtime library API.
//
// Semantics are exactly those of the interpreter (kernels.cu / DESIGN.md §3):
// the generator walks the same compiled schedule (steps, per-warp op lists,
// shared-memory slots and layouts) and emits, per op, the straight-line PTX
// the interpreter would have executed after decoding — offsets, widths,
// layouts and immediates become constants. Wide shifts by a variable amount
// call the interpreter's generic path (rtl_exec_wide, from jit_rt.ptx).
#include "jit.h"

#include <nvPTXCompiler.h>

#include <algorithm>
#include <array>
#include <atomic>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <iterator>
#include <sys/stat.h>
#include <unistd.h>
#include <mutex>
#include <sstream>
#include <map>
#include <thread>
#include <unordered_map>

namespace rtlsim {
namespace {

std::string fmt(const char *f, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, f);
  int n = vsnprintf(buf, sizeof buf, f, ap);
  va_end(ap);
  if (n < (int)sizeof buf) return std::string(buf, (size_t)std::max(n, 0));
  std::string s((size_t)n + 1, '\0');
  va_start(ap, f);
  vsnprintf(&s[0], s.size(), f, ap);
  va_end(ap);
  s.resize((size_t)n);
  return s;
}

// context values passed from the kernel to every step function
const char *kCtx32[] = {"smb", "lane", "wl", "N", "tbar", "mbar", "tmt"};
const char *kCtx64[] = {"tb_c0", "tb_c1", "tb_c2", "tb_c3", "tb_n0", "tb_n1", "tb_n2", "tb_n3",
                        "tb_x0", "tb_x1", "tb_x2", "tb_x3", "tb_i0", "tb_i1", "tb_i2", "tb_i3",
                        "outb", "dig", "wide", "smg", "bitl", "memb", "portb"};
constexpr int kN32 = 7, kN64 = 23;
constexpr uint64_t kTmemFwdOps = 8;   // forwarding budget of TMEM schedules (jit_fwd_ops)

// Split-phase step barrier (RTLSIM_JIT_SPLIT=1; default off, see below):
// instead of bar.sync at every step end, a warp arrives on an mbarrier (two,
// alternating by step parity) and, before waiting for the other warps, runs
// the next step's ops that cannot depend on them — operands written by this
// warp, or by other warps two or more steps earlier (not by a cp.async of
// another warp), destinations whose slot no other warp touched in the
// previous step. Measured cause (profiles/r02_ncu_c4_l16k2.txt): 54 % of the
// warp stall samples of a config-4 kernel at 16 op-lanes were the barrier.
// Off by default: ptxas treats code after a (non-.aligned) mbarrier.arrive as
// possibly divergent and duplicates blocks with divergence fallbacks around
// every vote.sync — config 3 SASS 195K -> 408K with the arrive alone — and
// only 18 % of the ops qualify as early (loads are late, 23 % read a value of
// the previous step, 17 % a value another warp loaded).
int jit_split() {
  const char *e = getenv("RTLSIM_JIT_SPLIT");
  return e ? atoi(e) : 0;
}

// Step barrier (RTLSIM_JIT_TBAR, read per build): 0 = one CTA-wide barrier
// per step (all K tiles x L op-lanes); 1 = a named barrier per tile (id
// 1 + tile, 32 L threads), so the tiles of a CTA do not wait for each other
// (with L == 1 a tile is one warp and the step edge is only a warp barrier);
// 2 = the CTA-wide barrier in its non-.aligned form (A/B, see the step loop).
// Measured on config 3 (profiles/r02_sweep_b.log): 1 is no faster than 0.
int jit_tbar() {
  const char *e = getenv("RTLSIM_JIT_TBAR");
  return e ? atoi(e) : 0;
}

// Shared-memory slot keys for register forwarding: (space, word offset).
enum : uint64_t { SP_W = 1, SP_H = 2, SP_B = 3, SP_S = 4 };   // [%rw] [%rh] [%rb] [%smb]
inline uint64_t skey(uint64_t sp, uint32_t off) { return (sp << 32) | off; }

// Writes of one step function, by (step, warp), per slot key (dry pass).
struct WriteLog {
  std::unordered_map<uint64_t, std::vector<std::pair<int32_t, uint32_t>>> w;
  std::unordered_map<uint64_t, std::vector<std::pair<int32_t, uint32_t>>> wo;   // of which opaque (cp.async / generic)
  // steps of the shared-memory reads of `key` (any warp), recorded by the
  // probe pass for dead slot-store elimination
  std::unordered_map<uint64_t, std::vector<int32_t>> rd;
  // a slot store of `key` in step s is dead when no shared-memory read of
  // the key lies in [s, next write step] (to the end if `to_end` and no later
  // write): every reader got the value from the writer's register
  bool dead_store(uint64_t key, int32_t s, bool to_end) const {
    int32_t nxt = INT32_MAX;
    auto it = w.find(key);
    if (it != w.end())
      for (const auto &x : it->second)
        if (x.first > s && x.first < nxt) nxt = x.first;
    if (nxt == INT32_MAX && !to_end) return false;
    auto r = rd.find(key);
    if (r == rd.end()) return true;
    for (int32_t t : r->second)
      if (t >= s && t <= nxt) return false;
    return true;
  }
  // another warp wrote `key` in steps (s0, s1]
  bool other(uint64_t key, uint32_t warp, int32_t s0, int32_t s1) const {
    auto it = w.find(key);
    if (it == w.end()) return false;
    for (const auto &x : it->second)
      if (x.second != warp && x.first > s0 && x.first <= s1) return true;
    return false;
  }
};

struct Em {
  std::string s;
  bool dig = false;   // emit the per-(stimulus, cycle) digest code (check-mode kernels only)
  // register forwarding of slot values within one step function: a slot this
  // warp stored (or already loaded) is read from the register that holds it,
  // unless another warp (or a cp.async / the generic wide path) wrote the slot
  // since. Stores are always kept (other warps / later functions read them).
  bool dry = true;           // dry pass: only record writes
  WriteLog *log = nullptr;
  bool probe = false;        // probe pass: record shared-memory reads in log->rd
  bool dse = false;          // drop dead slot stores (final pass, after a probe)
  bool to_end = false;       // this function runs to the end of the partition
  int32_t step = 0;
  uint32_t warp = 0;
  int32_t fwd_max = 0;       // forwarding distance in steps (0: off)
  struct Fwd {
    std::string reg;
    int32_t step;
    uint64_t op;               // op counter at the write (register-budget forwarding)
  };
  uint64_t opn = 0;            // descriptors emitted so far in this pass
  uint64_t fwd_ops = UINT64_MAX;   // forward only within this many ops (register budget)
  // ---- slot compaction (one op-lane): every value written to a slot is an
  // instance living from its defining step to its last shared-memory read;
  // only instances read back from shared memory (or written opaquely by
  // cp.async / the generic path) get space, allocated between the probe pass
  // and the final pass; the final pass emits the compacted offsets.
  struct Inst {
    uint32_t off, words;       // original slot words [off, off + words)
    int32_t s0, s1;            // defining step, last shared-memory read step
    bool need;                 // read from shared memory or written opaquely
    bool opq;                  // written opaquely (cp.async load / generic path)
    uint32_t nb;               // compacted offset (final pass)
  };
  bool compact = false;
  std::vector<Inst> *inst = nullptr;        // shared by the probe and final passes
  uint32_t ninst = 0;                       // instances begun in this pass
  std::unordered_map<uint64_t, uint32_t> cur;   // row key -> current instance
  std::vector<WideRec> *wrec = nullptr;     // generic-path records with compacted offsets
  std::vector<uint32_t> *bittab = nullptr;  // bit-op batch table (uint4 per op)
  std::unordered_map<uint64_t, std::vector<std::string>> vpend;   // wide groups awaiting their vector store
  std::unordered_map<uint64_t, Fwd> fwd;
  uint32_t nr = 0, nrd = 0, np = 0, nlab = 0;
  // N_pad the code is specialised for (0: generic, row stride from %N at run
  // time). Specialised code addresses a state row as [window + immediate]:
  // one 64-bit window register per arena base stays valid across the rows
  // within the ±8 MB immediate range of LDGSTS/STG (no IMAD.WIDE + IADD3 +
  // IADD3.X per access). Windows live within one basic block (cleared at
  // every label) so each use is dominated by its definition.
  uint32_t nspec = 0;
  bool used_v = false;         // (r2) 16-byte wide-register loads used (prologue sets %vsm / %vdl)
  bool ubase = false;          // (r2) arena windows from the kernel's params + %to<k> (inline bodies)
  std::map<std::string, std::pair<std::string, int64_t>> win;   // base -> (reg, row)
  std::string R() { return fmt("%%r%u", nr++); }
  std::string RD() { return fmt("%%rd%u", nrd++); }
  std::string P() { return fmt("%%p%u", np++); }
  std::string L(const char *pfx) { return fmt("$%s%u", pfx, nlab++); }
  void l(const std::string &x) {
    s += '\t';
    s += x;
    s += ";\n";
  }
  void lab(const std::string &x) {
    win.clear();
    s += x;
    s += ":\n";
  }
};

inline uint32_t mask_of(uint32_t w) { return w >= 32 ? 0xFFFFFFFFu : ((1u << w) - 1u); }

// Global address of `row` in the arena at base register `base` whose row
// stride is `sreg` (N4 / N2 / N / Nb bytes): "reg" or "reg+imm" for [..].
std::string gaddr(Em &e, const char *sreg, uint32_t row, const char *base) {
  if (!e.nspec) {
    std::string a = e.RD();
    e.l(fmt("mad.wide.u32 %s, %%%s, %u, %%%s", a.c_str(), sreg, row, base));
    return a;
  }
  const int64_t n = e.nspec;
  const int64_t stride = !strcmp(sreg, "N4") ? 4 * n : !strcmp(sreg, "N2") ? 2 * n : !strcmp(sreg, "N") ? n : n / 8;
  const int64_t lim = (1 << 23) - 64;   // signed 24-bit immediate, margin for the access width
  auto off_str = [](const std::string &r, int64_t off) {
    return off ? fmt("%s+%lld", r.c_str(), (long long)off) : r;
  };
  auto it = e.win.find(base);
  if (it != e.win.end()) {
    const int64_t off = ((int64_t)row - it->second.second) * stride;
    if (off >= -lim && off < lim) return off_str(it->second.first, off);
  }
  // new window: this row plus the rows up to ~12 MB above and ~4 MB below it
  const int64_t wrow = (int64_t)row + std::max<int64_t>(0, ((int64_t)1 << 22) / stride);
  std::string a = e.RD();
  if (e.ubase && !strncmp(base, "tb_", 3) && strlen(base) == 5 && strchr("cnxi", base[3])) {
    // (r2) uniform arena base from the kernel parameters (constant bank) plus
    // the thread's 64-bit class offset: no per-arena base register stays live
    const uint32_t ai = (uint32_t)(strchr("cnxi", base[3]) - "cnxi"), k = (uint32_t)(base[4] - '0');
    std::string u = e.RD(), t = e.RD();
    e.l(fmt("ld.param.u64 %s, [prm+%u]", u.c_str(), 32u * ai + 8u * k));
    e.l(fmt("add.s64 %s, %s, %%to%u", t.c_str(), u.c_str(), k));
    e.l(fmt("add.s64 %s, %s, %lld", a.c_str(), t.c_str(), (long long)(wrow * stride)));
  } else {
    e.l(fmt("add.s64 %s, %%%s, %lld", a.c_str(), base, (long long)(wrow * stride)));
  }
  e.win[base] = {a, wrow};
  return off_str(a, ((int64_t)row - wrow) * stride);
}

// words of one row (the unit a slot key addresses) per space
inline uint32_t sp_row_words(uint64_t sp) { return sp == SP_W ? 32u : sp == SP_H ? 16u : sp == SP_B ? 8u : 1u; }

// A value of `rows` rows (row keys off, off + stride, ...) is about to be
// written: start its instance (compaction). Safe at the start of a
// descriptor: the schedule never gives a value the slot of an operand that is
// still live in the same step.
void begin_value(Em &e, uint64_t sp, uint32_t off, uint32_t rows, bool opaque = false) {
  if (!e.compact || e.dry) return;
  const uint32_t stride = sp == SP_W ? 32u : 1u;
  const uint32_t id = e.ninst++;
  if (e.probe) {
    if (e.inst->size() <= id) e.inst->resize(id + 1);
    (*e.inst)[id] = Em::Inst{off, stride * (rows - 1) + sp_row_words(sp), e.step, e.step, opaque, opaque, 0};
  }
  for (uint32_t i = 0; i < rows; i++) e.cur[skey(sp, off + stride * i)] = id;
}
// the instance holding row key (sp, off), or -1 (never written: keep the offset)
int64_t inst_of(Em &e, uint64_t sp, uint32_t off) {
  if (!e.compact || e.dry) return -1;
  auto it = e.cur.find(skey(sp, off));
  return it == e.cur.end() ? -1 : (int64_t)it->second;
}
// a shared-memory read of row (sp, off): extends the instance (probe pass)
void inst_read(Em &e, uint64_t sp, uint32_t off) {
  const int64_t id = inst_of(e, sp, off);
  if (id < 0 || !e.probe) return;
  Em::Inst &I = (*e.inst)[(size_t)id];
  I.need = true;
  I.s1 = std::max(I.s1, e.step);
}
// the word offset to emit for row (sp, off)
uint32_t xoff(Em &e, uint64_t sp, uint32_t off) {
  const int64_t id = inst_of(e, sp, off);
  if (id < 0 || e.probe) return off;
  const Em::Inst &I = (*e.inst)[(size_t)id];
  return I.nb + (off - I.off);
}

const char *kSpBase[5] = {"", "%rw", "%rh", "%rb", "%smb"};
const char *kSpTy[5] = {"", "u32", "u16", "u8", "u32"};

// slot read (forwarded from a register when valid)
std::string lds(Em &e, uint64_t sp, uint32_t off) {
  const uint64_t k = skey(sp, off);
  if (!e.dry && e.fwd_max > 0) {
    auto it = e.fwd.find(k);
    if (it != e.fwd.end()) {
      if (e.step - it->second.step <= e.fwd_max && e.opn - it->second.op <= e.fwd_ops &&
          !e.log->other(k, e.warp, it->second.step, e.step))
        return it->second.reg;
      e.fwd.erase(it);
    }
  }
  std::string r = e.R();
  if (sp == SP_W && in_tmem(off)) {
    // (r2) TMEM word: column (off - base) / 32 of this tile's lane quarter
    e.l(fmt("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%s}, [%%tmt+%u]", r.c_str(), (off - kTmemBase) / 32u));
    e.l("tcgen05.wait::ld.sync.aligned");
  } else {
    e.l(fmt("ld.shared.%s %s, [%s+%u]", kSpTy[sp], r.c_str(), kSpBase[sp], xoff(e, sp, off) * 4));
  }
  if (e.probe) e.log->rd[k].push_back(e.step);
  inst_read(e, sp, off);
  // a read-created entry is only as good as the read itself: a write by
  // another warp in this same step is not ordered with it, so the validity
  // window starts one step earlier
  if (!e.dry) e.fwd[k] = Em::Fwd{r, e.step - 1, e.opn};
  return r;
}
// slot write from a register
void sts(Em &e, uint64_t sp, uint32_t off, const std::string &r) {
  const uint64_t k = skey(sp, off);
  const int64_t id = inst_of(e, sp, off);
  const bool unread = id >= 0 && !e.probe && !(*e.inst)[(size_t)id].need;   // compacted away
  if (!unread && !(e.dse && e.log->dead_store(k, e.step, e.to_end))) {
    if (sp == SP_W && in_tmem(off))
      e.l(fmt("tcgen05.st.sync.aligned.32x32b.x1.b32 [%%tmt+%u], {%s}", (off - kTmemBase) / 32u, r.c_str()));
    else
      e.l(fmt("st.shared.%s [%s+%u], %s", kSpTy[sp], kSpBase[sp], xoff(e, sp, off) * 4, r.c_str()));
  }
  if (e.dry) e.log->w[k].push_back({e.step, e.warp});
  else e.fwd[k] = Em::Fwd{r, e.step, e.opn};
}
// ----------------------------------------------- vector layout of wide values --
// (r2, RTLSIM_JIT_VWIDE=1, default OFF: on the B200 it failed parity — a
// misaligned-address fault and wrong config-3 golden digests — for a 1 %
// config-4 gain; kept as an option until fixed) A value of >= 2 words in a U32 slot is
// laid out in groups of up to 4 words: group g (words 4g..4g+gs-1, gs =
// min(4, nw - 4g)) occupies 32 lanes x gs words at byte 16 * 32 * g of the
// slot, lane l's words contiguous — one LDS.128 / STS.128 (LDS.64 for a pair)
// moves a lane's whole group, where the row layout needs one instruction per
// word. Same slot size; keys stay (SP_W, off + 32 i) per word. Only the JIT
// uses it (the interpreter keeps rows); variable wide shifts are emitted
// inline (no generic call reading the row layout).
bool jit_vwide() {
  static const bool on = getenv("RTLSIM_JIT_VWIDE") && atoi(getenv("RTLSIM_JIT_VWIDE")) != 0;
  return on;
}
bool is_vwide(uint32_t lay, uint32_t w) { return jit_vwide() && lay == LC_U32 && nwords(w) >= 2; }
const char *kLaneBase[5] = {"", "%rw", "%rq2", "%rq3", "%rq4"};
uint32_t vgs(uint32_t nw, uint32_t g) { return std::min<uint32_t>(4u, nw - 4u * g); }
// byte offset of word i of the wide value at slot off (from the lane base of its group size)
uint32_t vbyte(Em &e, uint32_t off, uint32_t nw, uint32_t i) {
  return xoff(e, SP_W, off) * 4u + 512u * (i / 4u) + 4u * (i % 4u);
}
// a still-valid forwarded register for key, or ""
std::string fwd_get(Em &e, uint64_t k) {
  if (e.dry || e.fwd_max <= 0) return "";
  auto it = e.fwd.find(k);
  if (it == e.fwd.end()) return "";
  if (e.step - it->second.step <= e.fwd_max && e.opn - it->second.op <= e.fwd_ops &&
      !e.log->other(k, e.warp, it->second.step, e.step))
    return it->second.reg;
  e.fwd.erase(it);
  return "";
}
// word i of the wide value at slot off (nw words): forwarded, or its group loaded at once
std::string vword(Em &e, uint32_t off, uint32_t nw, uint32_t i) {
  const uint64_t k = skey(SP_W, off + 32u * i);
  std::string r = fwd_get(e, k);
  if (!r.empty()) return r;
  const uint32_t g = i / 4u, gs = vgs(nw, g);
  if (gs == 1 || gs == 3) {   // no vector width: only the word asked for
    r = e.R();
    e.l(fmt("ld.shared.u32 %s, [%s+%u]", r.c_str(), kLaneBase[gs], vbyte(e, off, nw, i)));
    if (e.probe) e.log->rd[k].push_back(e.step);
    inst_read(e, SP_W, off + 32u * i);
    if (!e.dry) e.fwd[k] = Em::Fwd{r, e.step - 1, e.opn};
    return r;
  }
  std::string regs[4];
  for (uint32_t j = 0; j < gs; j++) regs[j] = e.R();
  const uint32_t b = vbyte(e, off, nw, 4u * g);
  if (gs == 4) {
    e.l(fmt("ld.shared.v4.u32 {%s, %s, %s, %s}, [%%rq4+%u]", regs[0].c_str(), regs[1].c_str(), regs[2].c_str(),
            regs[3].c_str(), b));
  } else {
    e.l(fmt("ld.shared.v2.u32 {%s, %s}, [%%rq2+%u]", regs[0].c_str(), regs[1].c_str(), b));
  }
  for (uint32_t j = 0; j < gs; j++) {
    const uint64_t kj = skey(SP_W, off + 32u * (4u * g + j));
    if (e.probe) e.log->rd[kj].push_back(e.step);
    inst_read(e, SP_W, off + 32u * (4u * g + j));
    if (!e.dry) e.fwd[kj] = Em::Fwd{regs[j], e.step - 1, e.opn};
  }
  return regs[i % 4u];
}
// word i of a wide result: buffered until its group is complete, then one
// vector store (kept when any word of the group is read back from shared memory)
void vstore(Em &e, uint32_t off, uint32_t nw, uint32_t i, const std::string &v) {
  const uint32_t g = i / 4u, gs = vgs(nw, g);
  auto &pend = e.vpend[((uint64_t)off << 8) | g];
  if (pend.size() < gs) pend.resize(gs);
  pend[i % 4u] = v;
  const uint64_t k = skey(SP_W, off + 32u * i);
  if (e.dry) e.log->w[k].push_back({e.step, e.warp});
  else e.fwd[k] = Em::Fwd{v, e.step, e.opn};
  for (uint32_t j = 0; j < gs; j++)
    if (pend[j].empty()) return;
  bool live = false;
  for (uint32_t j = 0; j < gs; j++) {
    const uint64_t kj = skey(SP_W, off + 32u * (4u * g + j));
    const int64_t id = inst_of(e, SP_W, off + 32u * (4u * g + j));
    const bool unread = id >= 0 && !e.probe && !(*e.inst)[(size_t)id].need;
    if (!unread && !(e.dse && e.log->dead_store(kj, e.step, e.to_end))) live = true;
  }
  if (live) {
    const uint32_t b = vbyte(e, off, nw, 4u * g);
    if (gs == 4)
      e.l(fmt("st.shared.v4.u32 [%%rq4+%u], {%s, %s, %s, %s}", b, pend[0].c_str(), pend[1].c_str(), pend[2].c_str(),
              pend[3].c_str()));
    else if (gs == 2)
      e.l(fmt("st.shared.v2.u32 [%%rq2+%u], {%s, %s}", b, pend[0].c_str(), pend[1].c_str()));
    else
      for (uint32_t j = 0; j < gs; j++) e.l(fmt("st.shared.u32 [%s+%u], %s", kLaneBase[gs], b + 4u * j, pend[j].c_str()));
  }
  e.vpend.erase(((uint64_t)off << 8) | g);
}

// a write this warp cannot forward (cp.async, generic path)
void opaque_write(Em &e, uint64_t sp, uint32_t off) {
  const uint64_t k = skey(sp, off);
  if (e.dry) {
    e.log->w[k].push_back({e.step, e.warp});
    e.log->wo[k].push_back({e.step, e.warp});
  }
  else e.fwd.erase(k);
  const int64_t id = inst_of(e, sp, off);
  if (id >= 0 && e.probe) (*e.inst)[(size_t)id].need = true;
}
uint64_t layout_space(uint32_t lay) {
  return lay == LC_U32 ? SP_W : lay == LC_U16 ? SP_H : lay == LC_U8 ? SP_B : SP_S;
}
// a shared-memory read that bypasses lds (direct loads, the generic path)
void note_read(Em &e, uint64_t sp, uint32_t off) {
  if (e.probe) e.log->rd[skey(sp, off)].push_back(e.step);
  inst_read(e, sp, off);
}
// every slot word an operand (offset, width, layout) of the generic path may read
void note_operand_reads(Em &e, uint32_t off, uint32_t w, uint32_t lay) {
  if (lay == LC_IMM || w == 0) return;
  const uint64_t sp = layout_space(lay);
  for (uint32_t i = 0; i < nwords(w); i++) note_read(e, sp, sp == SP_W ? off + 32 * i : off + i);
}

// ------------------------------------------------------------- operands --
// narrow (<= 32-bit) value from a slot of layout `lay` (or an immediate)
std::string fetch_narrow(Em &e, uint32_t lay, uint32_t off, uint32_t /*w*/) {
  switch (lay) {
    case LC_U32: return lds(e, SP_W, off);
    case LC_U16: return lds(e, SP_H, off);
    case LC_U8: return lds(e, SP_B, off);
    case LC_BIT: {
      std::string t = lds(e, SP_S, off), t2 = e.R(), r = e.R();
      e.l(fmt("shr.b32 %s, %s, %%lane", t2.c_str(), t.c_str()));
      e.l(fmt("and.b32 %s, %s, 1", r.c_str(), t2.c_str()));
      return r;
    }
    case LC_BCAST: return lds(e, SP_S, off);
    default: {   // LC_IMM
      std::string r = e.R();
      e.l(fmt("mov.u32 %s, %u", r.c_str(), off));
      return r;
    }
  }
}

void store_narrow(Em &e, uint32_t lay, uint32_t off, const std::string &r) {
  switch (lay) {
    case LC_U32: sts(e, SP_W, off, r); break;
    case LC_U16: sts(e, SP_H, off, r); break;
    case LC_U8: sts(e, SP_B, off, r); break;
    default: {   // LC_BIT: pack the warp's 32 results
      std::string p = e.P(), m = e.R();
      e.l(fmt("setp.ne.u32 %s, %s, 0", p.c_str(), r.c_str()));
      e.l(fmt("vote.sync.ballot.b32 %s, %s, 0xffffffff", m.c_str(), p.c_str()));
      // every lane holds the same ballot word: an unpredicated store is one
      // same-address wavefront (and compiles much faster than a predicated one)
      sts(e, SP_S, off, m);
      break;
    }
  }
}

// sign-extend a canonical w-bit value held in r (w < 32) to 32 bits
std::string sext32(Em &e, const std::string &r, uint32_t w) {
  if (w >= 32) return r;
  std::string t = e.R(), u = e.R();
  e.l(fmt("shl.b32 %s, %s, %u", t.c_str(), r.c_str(), 32 - w));
  e.l(fmt("shr.s32 %s, %s, %u", u.c_str(), t.c_str(), 32 - w));
  return u;
}

// a wide-op operand: word i of the value zero- or sign-extended
struct WOp {
  uint32_t off = 0, w = 0, lay = LC_U32;
  std::vector<std::string> zw, sw;   // cached zero / sign views per word
  std::string top_sx;                // sign-extended top word
  std::string fill;                  // 0 / all ones from the sign
  std::string narrow;                // fetched value when w <= 32
};

std::string wword(Em &e, WOp &o, uint32_t i, bool sx) {
  const uint32_t n = nwords(o.w), rem = o.w & 31u;
  if (o.zw.size() < n) {
    o.zw.assign(n, "");
    o.sw.assign(n, "");
  }
  auto raw = [&](uint32_t j) -> std::string {
    if (!o.zw[j].empty()) return o.zw[j];
    std::string r;
    if (o.w <= 32) {
      if (o.narrow.empty()) o.narrow = fetch_narrow(e, o.lay, o.off, o.w);
      r = o.narrow;
    } else if (is_vwide(o.lay, o.w)) {
      r = vword(e, o.off, n, j);
    } else {
      r = o.lay == LC_BCAST ? lds(e, SP_S, o.off + j) : lds(e, SP_W, o.off + 32 * j);
    }
    o.zw[j] = r;
    return r;
  };
  if (i < n) {
    if (!sx || i != n - 1 || rem == 0) return raw(i);
    if (o.top_sx.empty()) o.top_sx = sext32(e, raw(n - 1), rem);
    return o.top_sx;
  }
  if (!sx) return "0";
  if (o.fill.empty()) {
    std::string top = (rem == 0) ? raw(n - 1) : (o.top_sx.empty() ? (o.top_sx = sext32(e, raw(n - 1), rem)) : o.top_sx);
    o.fill = e.R();
    e.l(fmt("shr.s32 %s, %s, 31", o.fill.c_str(), top.c_str()));
  }
  return o.fill;
}

// (r2) word i of a wide result held in TMEM: buffered until all n words are
// there, then runs of live (not dead-store-eliminated) consecutive columns
// go out as vector tcgen05.st (.x2 .. .x32)
void tm_vstore(Em &e, uint32_t off, uint32_t n, uint32_t i, const std::string &v) {
  auto &pend = e.vpend[((uint64_t)off << 8) | 0xFFu];
  if (pend.size() < n) pend.resize(n);
  pend[i] = v;
  const uint64_t k = skey(SP_W, off + 32u * i);
  if (e.dry) e.log->w[k].push_back({e.step, e.warp});
  else e.fwd[k] = Em::Fwd{v, e.step, e.opn};
  for (uint32_t j = 0; j < n; j++)
    if (pend[j].empty()) return;
  std::vector<char> live(n, 1);
  for (uint32_t j = 0; j < n; j++)
    live[j] = !(e.dse && e.log->dead_store(skey(SP_W, off + 32u * j), e.step, e.to_end));
  const uint32_t c0 = (off - kTmemBase) / 32u;
  for (uint32_t j = 0; j < n;) {
    if (!live[j]) {
      j++;
      continue;
    }
    uint32_t m = j + 1;
    while (m < n && live[m]) m++;
    uint32_t c = c0 + j, rem = m - j, w = j;
    while (rem) {
      uint32_t cnt = 1;
      while (cnt * 2 <= rem && cnt * 2 <= 32u && (c % (cnt * 2)) == 0) cnt *= 2;
      std::string regs;
      for (uint32_t t = 0; t < cnt; t++) regs += (t ? ", " : "") + pend[w + t];
      e.l(fmt("tcgen05.st.sync.aligned.32x32b.x%u.b32 [%%tmt+%u], {%s}", cnt, c, regs.c_str()));
      c += cnt;
      w += cnt;
      rem -= cnt;
    }
    j = m;
  }
  e.vpend.erase(((uint64_t)off << 8) | 0xFFu);
}

// store word i of a wide result (masking the top word)
void wstore(Em &e, uint32_t off, uint32_t wd, uint32_t i, const std::string &v) {
  const uint32_t n = nwords(wd), rem = wd & 31u;
  std::string x = v;
  if (v == "0") {
    x = e.R();
    e.l(fmt("mov.u32 %s, 0", x.c_str()));
  }
  if (wd <= 32) {   // a narrow result of a wide op
    std::string m = x;
    if (wd < 32) {
      m = e.R();
      e.l(fmt("and.b32 %s, %s, %u", m.c_str(), x.c_str(), mask_of(wd)));
    }
    store_narrow(e, value_layout(wd, false), off, m);
    return;
  }
  if (i == n - 1 && rem) {
    std::string m = e.R();
    e.l(fmt("and.b32 %s, %s, %u", m.c_str(), x.c_str(), mask_of(rem)));
    x = m;
  }
  if (in_tmem(off) && n >= 2) tm_vstore(e, off, n, i, x);
  else if (jit_vwide()) vstore(e, off, n, i, x);
  else sts(e, SP_W, off + 32 * i, x);
}

std::string reg_of(Em &e, const std::string &v) {
  if (v == "0") {
    std::string r = e.R();
    e.l(fmt("mov.u32 %s, 0", r.c_str()));
    return r;
  }
  return v;
}

// -------------------------------------------------------- memories --
// word t of entry idx (a register holding the lane's canonical index) of
// memory m: 0 when idx >= depth. Memory rows are [row][N_pad] u32; %memb is
// this stimulus' column. The rows differ per lane, so the load is a gather.
thread_local const Program *t_prog = nullptr;   // the program being emitted (memory shapes)
std::string emit_mem_read(Em &e, const std::string &idx, uint32_t m, uint32_t t) {
  const Program &G = *t_prog;
  const uint32_t nw = nwords(G.mem_width[m]), row = G.mem_row0[m] + t;
  std::string p = e.P(), off = e.RD(), a = e.RD(), v = e.R();
  e.l(fmt("setp.lt.u32 %s, %s, %u", p.c_str(), idx.c_str(), G.mem_depth[m]));
  if (e.nspec) {
    const uint64_t n4 = 4ull * e.nspec;
    e.l(fmt("mul.wide.u32 %s, %s, %llu", off.c_str(), idx.c_str(), (unsigned long long)(n4 * nw)));
    e.l(fmt("add.s64 %s, %s, %llu", a.c_str(), off.c_str(), (unsigned long long)(n4 * row)));
  } else {
    std::string k = e.R(), r = e.R();
    e.l(fmt("mul.lo.u32 %s, %%N4, %u", k.c_str(), nw));
    e.l(fmt("mul.wide.u32 %s, %s, %s", off.c_str(), idx.c_str(), k.c_str()));
    e.l(fmt("mul.wide.u32 %s, %%N4, %u", a.c_str(), row));
    e.l(fmt("add.s64 %s, %s, %s", a.c_str(), a.c_str(), off.c_str()));
  }
  e.l(fmt("add.s64 %s, %s, %%memb", a.c_str(), a.c_str()));
  e.l(fmt("mov.u32 %s, 0", v.c_str()));
  e.l(fmt("@%s ld.global.u32 %s, [%s]", p.c_str(), v.c_str(), a.c_str()));
  return v;
}

// -------------------------------------------------------- narrow ops --
void emit_narrow(Em &e, const Desc &q) {
  const uint32_t op = q.x & 0xFFu;
  const uint32_t la = (q.x >> 8) & 7u, lb = (q.x >> 11) & 7u, lc = (q.x >> 14) & 7u, ld = (q.x >> 17) & 7u;
  const uint32_t wd = (q.x >> 20) & 63u, wa = q.x >> 26, wb = q.w & 63u, imm = (q.w >> 6) & 31u;
  const bool hb = (q.w >> 11) & 1u, hc = (q.w >> 12) & 1u;
  const uint32_t d = q.y & 0xFFFFu, a = q.y >> 16, b = q.z & 0xFFFFu, c = q.z >> 16;
  begin_value(e, layout_space(ld), d, 1);
  if (op == RTLSIM_OP_MEMRD) {   // ARRSEL read: entry V[a] of memory q.z (reading 12)
    std::string idx = fetch_narrow(e, la, a, wa);
    std::string v = emit_mem_read(e, idx, q.z, 0);
    store_narrow(e, ld, d, v);
    return;
  }
  if (op == RTLSIM_OP_MUX && la == LC_BIT && hb && hc) {
    // 1-bit select straight from its packed word: the lane's bit moved to
    // bit 31 and sign-filled is the all-ones / zero mask of the LOP3 mux
    std::string t = lds(e, SP_S, a), y = fetch_narrow(e, lb, b, wb), z = fetch_narrow(e, lc, c, 32);
    std::string m1 = e.R(), m = e.R(), r = e.R();
    e.l(fmt("shl.b32 %s, %s, %%lsh", m1.c_str(), t.c_str()));
    e.l(fmt("shr.s32 %s, %s, 31", m.c_str(), m1.c_str()));
    e.l(fmt("lop3.b32 %s, %s, %s, %s, 0xca", r.c_str(), m.c_str(), y.c_str(), z.c_str()));
    std::string res = r;
    if (wd < 32) {
      res = e.R();
      e.l(fmt("and.b32 %s, %s, %u", res.c_str(), r.c_str(), mask_of(wd)));
    }
    store_narrow(e, ld, d, res);
    return;
  }
  std::string x = fetch_narrow(e, la, a, wa);
  std::string y = hb ? fetch_narrow(e, lb, b, wb) : std::string();
  std::string z = hc ? fetch_narrow(e, lc, c, 32) : std::string();
  // a 1-bit compare / reduction into a packed bit slot: predicate -> ballot
  // directly (no 0/1 materialisation, no second test)
  if (ld == LC_BIT) {
    const char *cc = nullptr;
    bool sg = false;
    std::string u = x, v = y;
    switch (op) {
      case RTLSIM_OP_EQ: cc = "eq"; break;
      case RTLSIM_OP_NE: cc = "ne"; break;
      case RTLSIM_OP_LTU: cc = "lt"; break;
      case RTLSIM_OP_LEU: cc = "le"; break;
      case RTLSIM_OP_GTU: cc = "gt"; break;
      case RTLSIM_OP_GEU: cc = "ge"; break;
      case RTLSIM_OP_LTS: cc = "lt"; sg = true; break;
      case RTLSIM_OP_LES: cc = "le"; sg = true; break;
      case RTLSIM_OP_GTS: cc = "gt"; sg = true; break;
      case RTLSIM_OP_GES: cc = "ge"; sg = true; break;
      case RTLSIM_OP_REDAND: cc = "eq"; v = fmt("%u", mask_of(wa)); break;
      case RTLSIM_OP_REDOR: cc = "ne"; v = "0"; break;
      default: break;
    }
    if (cc) {
      if (sg) {
        u = sext32(e, x, wa);
        v = sext32(e, y, wb);
      }
      std::string p = e.P(), m = e.R();
      e.l(fmt("setp.%s.%s %s, %s, %s", cc, sg ? "s32" : "u32", p.c_str(), u.c_str(), v.c_str()));
      e.l(fmt("vote.sync.ballot.b32 %s, %s, 0xffffffff", m.c_str(), p.c_str()));
      sts(e, SP_S, d, m);
      return;
    }
  }
  std::string r = e.R();
  bool canon = false;   // result already < 2^wd
  // bits the raw result can occupy (operands are canonical: < 2^w); no mask
  // is needed when they fit wd. (A byte / half-word slot store would truncate
  // an 8- / 16-bit value by itself, but the register is forwarded to later
  // reads, so it must be canonical too.)
  uint32_t span = 32;
  switch (op) {
    case RTLSIM_OP_COPY: case RTLSIM_OP_SHRL: case RTLSIM_OP_DIVU: case RTLSIM_OP_MODU: span = wa; break;
    case RTLSIM_OP_AND: span = std::min(wa, wb); break;
    case RTLSIM_OP_OR: case RTLSIM_OP_XOR: span = std::max(wa, wb); break;
    case RTLSIM_OP_ADD: span = std::max(wa, wb) + 1; break;
    case RTLSIM_OP_MUL: span = wa + wb; break;
    case RTLSIM_OP_CONCAT: span = wa + wb; break;
    case RTLSIM_OP_SLICE: span = wa > imm ? wa - imm : 0; break;
    default: break;
  }
  if (span <= wd) canon = true;
  // predicate-free forms (set.* gives 0 / all ones): ptxas compiles them far
  // faster than setp/selp chains and the SASS is the same length
  auto cmp = [&](const char *cc, const std::string &u, const std::string &v) {
    std::string m = e.R();
    const char *ty = strstr(cc, ".s32") ? "s32" : "u32";
    std::string c2(cc);
    c2 = c2.substr(0, c2.find('.'));
    e.l(fmt("set.%s.u32.%s %s, %s, %s", c2.c_str(), ty, m.c_str(), u.c_str(), v.c_str()));
    e.l(fmt("and.b32 %s, %s, 1", r.c_str(), m.c_str()));
    canon = true;
  };
  switch (op) {
    case RTLSIM_OP_COPY: e.l(fmt("mov.u32 %s, %s", r.c_str(), x.c_str())); break;
    case RTLSIM_OP_SEXT: e.l(fmt("mov.u32 %s, %s", r.c_str(), sext32(e, x, wa).c_str())); break;
    case RTLSIM_OP_NOT: e.l(fmt("not.b32 %s, %s", r.c_str(), x.c_str())); break;
    case RTLSIM_OP_AND: e.l(fmt("and.b32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_OR: e.l(fmt("or.b32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_XOR: e.l(fmt("xor.b32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_ADD: e.l(fmt("add.u32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_SUB: e.l(fmt("sub.u32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_NEG: e.l(fmt("neg.s32 %s, %s", r.c_str(), x.c_str())); break;
    case RTLSIM_OP_MUL: e.l(fmt("mul.lo.u32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;
    case RTLSIM_OP_DIVU:
    case RTLSIM_OP_MODU: {   // b == 0 gives 0
      std::string m = e.R(), t = e.R();
      e.l(fmt("set.ne.u32.u32 %s, %s, 0", m.c_str(), y.c_str()));
      e.l(fmt("%s.u32 %s, %s, %s", op == RTLSIM_OP_DIVU ? "div" : "rem", t.c_str(), x.c_str(), y.c_str()));
      e.l(fmt("and.b32 %s, %s, %s", r.c_str(), t.c_str(), m.c_str()));
      break;
    }
    case RTLSIM_OP_EQ: cmp("eq.u32", x, y); break;
    case RTLSIM_OP_NE: cmp("ne.u32", x, y); break;
    case RTLSIM_OP_LTU: cmp("lt.u32", x, y); break;
    case RTLSIM_OP_LEU: cmp("le.u32", x, y); break;
    case RTLSIM_OP_GTU: cmp("gt.u32", x, y); break;
    case RTLSIM_OP_GEU: cmp("ge.u32", x, y); break;
    case RTLSIM_OP_LTS: cmp("lt.s32", sext32(e, x, wa), sext32(e, y, wb)); break;
    case RTLSIM_OP_LES: cmp("le.s32", sext32(e, x, wa), sext32(e, y, wb)); break;
    case RTLSIM_OP_GTS: cmp("gt.s32", sext32(e, x, wa), sext32(e, y, wb)); break;
    case RTLSIM_OP_GES: cmp("ge.s32", sext32(e, x, wa), sext32(e, y, wb)); break;
    case RTLSIM_OP_SHL: {   // b >= wd gives 0
      std::string m = e.R(), t = e.R();
      e.l(fmt("set.lt.u32.u32 %s, %s, %u", m.c_str(), y.c_str(), wd));
      e.l(fmt("shl.b32 %s, %s, %s", t.c_str(), x.c_str(), y.c_str()));
      e.l(fmt("and.b32 %s, %s, %s", r.c_str(), t.c_str(), m.c_str()));
      break;
    }
    case RTLSIM_OP_SHRL: e.l(fmt("shr.u32 %s, %s, %s", r.c_str(), x.c_str(), y.c_str())); break;   // clamps at 32
    case RTLSIM_OP_SHRA: e.l(fmt("shr.s32 %s, %s, %s", r.c_str(), sext32(e, x, wa).c_str(), y.c_str())); break;
    case RTLSIM_OP_MUX: {   // m = all ones when sel != 0; r = (y & m) | (z & ~m)
      std::string m = e.R();
      e.l(fmt("set.ne.u32.u32 %s, %s, 0", m.c_str(), x.c_str()));
      e.l(fmt("lop3.b32 %s, %s, %s, %s, 0xca", r.c_str(), m.c_str(), y.c_str(), z.c_str()));
      break;
    }
    case RTLSIM_OP_CONCAT:
      if (wb >= 32) {
        e.l(fmt("mov.u32 %s, %s", r.c_str(), y.c_str()));
      } else {
        std::string t = e.R();
        e.l(fmt("shl.b32 %s, %s, %u", t.c_str(), x.c_str(), wb));
        e.l(fmt("or.b32 %s, %s, %s", r.c_str(), t.c_str(), y.c_str()));
      }
      break;
    case RTLSIM_OP_SLICE: e.l(fmt("shr.u32 %s, %s, %u", r.c_str(), x.c_str(), imm)); break;
    case RTLSIM_OP_REDAND: cmp("eq.u32", x, fmt("%u", mask_of(wa))); break;
    case RTLSIM_OP_REDOR: cmp("ne.u32", x, "0"); break;
    default: {   // REDXOR
      std::string t = e.R();
      e.l(fmt("popc.b32 %s, %s", t.c_str(), x.c_str()));
      e.l(fmt("and.b32 %s, %s, 1", r.c_str(), t.c_str()));
      canon = true;
      break;
    }
  }
  std::string res = r;
  if (!canon && wd < 32) {
    res = e.R();
    e.l(fmt("and.b32 %s, %s, %u", res.c_str(), r.c_str(), mask_of(wd)));
  }
  store_narrow(e, ld, d, res);
}

// ---------------------------------------------------------- wide ops --
void emit_generic_call(Em &e, uint32_t idx) {
  std::string rec = e.RD();
  e.l(fmt("add.u64 %s, %%wide, %u", rec.c_str(), idx * (uint32_t)sizeof(WideRec)));
  e.s += "\t{\n\t.param .b64 wp0;\n\t.param .b64 wp1;\n\t.param .b32 wp2;\n";
  e.l("st.param.b64 [wp0], %smg");
  e.l(fmt("st.param.b64 [wp1], %s", rec.c_str()));
  e.l("st.param.b32 [wp2], %lane");
  e.l("call.uni rtl_exec_wide, (wp0, wp1, wp2)");
  e.s += "\t}\n";
}
void generic_wide(Em &e, const WideRec &w, uint32_t idx) {
  if (getenv("RTLSIM_TMEM_DEBUG") && (in_tmem(w.a) || in_tmem(w.b) || in_tmem(w.c) || in_tmem(w.d)))
    fprintf(stderr, "generic wide op %u with a TMEM operand: d %x a %x b %x c %x wd %u wa %u wb %u lays %x\n", w.op,
            w.d, w.a, w.b, w.c, w.wd, w.wa, w.wb, w.lays);
  note_operand_reads(e, w.a, w.wa, w.lays & 0xFFu);
  note_operand_reads(e, w.b, w.wb, (w.lays >> 8) & 0xFFu);
  note_operand_reads(e, w.c, w.wc, (w.lays >> 16) & 0xFFu);
  if (e.compact && e.wrec) {
    // the generic path reads the record's slot offsets: a copy with the
    // compacted offsets, in this partition's own record table
    WideRec r = w;
    auto tr = [&](uint32_t off, uint32_t wv, uint32_t lay) -> uint32_t {
      if (lay == LC_IMM || wv == 0) return off;
      return xoff(e, layout_space(lay), off);
    };
    r.a = tr(w.a, w.wa, w.lays & 0xFFu);
    r.b = tr(w.b, w.wb, (w.lays >> 8) & 0xFFu);
    r.c = tr(w.c, w.wc, (w.lays >> 16) & 0xFFu);
    r.d = tr(w.d, w.wd, w.wd <= 32 ? value_layout(w.wd, false) : LC_U32);
    idx = (uint32_t)e.wrec->size();
    e.wrec->push_back(r);
  }
  emit_generic_call(e, idx);
  if (w.wd <= 32) {
    opaque_write(e, layout_space(value_layout(w.wd, false)), w.d);
  } else {
    for (uint32_t i = 0; i < nwords(w.wd); i++) opaque_write(e, SP_W, w.d + 32 * i);
  }
}

// SHL / SHRL / SHRA of a wide value by a variable amount, inline (vector
// layout): word i of the result is a funnel shift of the
// operand's words i -/+ q and i -/+ q + 1 (q = s / 32), read at run-time
// word indices (per lane) straight from shared memory.
void emit_vshift(Em &e, const WideRec &w, WOp &A, WOp &B) {
  const uint32_t op = w.op, wd = w.wd, nd = nwords(wd), wa = A.w, nwa = nwords(wa);
  const uint32_t Ws = std::max(wd, wa);
  const uint32_t limit = op == RTLSIM_OP_SHL ? wd : Ws;
  const bool sra = op == RTLSIM_OP_SHRA;
  // the shift amount, saturated to 2^32 - 1 when it does not fit 32 bits
  std::string sam = reg_of(e, wword(e, B, 0, false));
  if (nwords(B.w) > 1) {
    std::string hi = e.R();
    e.l(fmt("mov.u32 %s, 0", hi.c_str()));
    for (uint32_t i = 1; i < nwords(B.w); i++) {
      std::string t = e.R();
      e.l(fmt("or.b32 %s, %s, %s", t.c_str(), hi.c_str(), reg_of(e, wword(e, B, i, false)).c_str()));
      hi = t;
    }
    std::string p = e.P(), t = e.R();
    e.l(fmt("setp.ne.u32 %s, %s, 0", p.c_str(), hi.c_str()));
    e.l(fmt("selp.u32 %s, -1, %s, %s", t.c_str(), sam.c_str(), p.c_str()));
    sam = t;
  }
  // operand kind: 0 = a narrow value (a0), 1 = broadcast constant words, 2 = vector layout
  uint32_t kind = 0, abase = 0;
  std::string a0 = "0", fill = "0";
  if (wa <= 32) {
    a0 = reg_of(e, wword(e, A, 0, sra));
  } else if (A.lay == LC_BCAST) {
    kind = 1;
    abase = xoff(e, SP_S, A.off) * 4;
    for (uint32_t i = 0; i < nwa; i++) note_read(e, SP_S, A.off + i);
  } else {
    kind = 2;
    abase = xoff(e, SP_W, A.off) * 4;
    for (uint32_t i = 0; i < nwa; i++) note_read(e, SP_W, A.off + 32 * i);
  }
  if (sra) fill = reg_of(e, wword(e, A, nwa, true));   // the sign word (top word sign-extended)
  std::string top = (kind != 0 && sra && (wa & 31u)) ? reg_of(e, wword(e, A, nwa - 1, true)) : std::string("0");
  // the loop lives in rtl_vshift (one copy per module): its code is fetched once
  e.s += "\t{\n";
  const char *pn[] = {"vs_op", "vs_nd", "vs_rem", "vs_nwa", "vs_kind", "vs_ab", "vs_a0", "vs_s", "vs_lim",
                      "vs_fill", "vs_db", "vs_top"};
  std::string ab = e.R(), db = e.R();   // absolute shared addresses (lane 0 / word 0)
  e.l(fmt("add.u32 %s, %%smb, %u", ab.c_str(), abase));
  e.l(fmt("add.u32 %s, %%smb, %u", db.c_str(), xoff(e, SP_W, w.d) * 4));
  const std::string pv[] = {fmt("%u", op), fmt("%u", nd), fmt("%u", wd & 31u), fmt("%u", nwa), fmt("%u", kind),
                            ab, a0, sam, fmt("%u", limit), fill, db, top};
  for (int i = 0; i < 12; i++) {
    e.s += fmt("\t.param .b32 %s;\n", pn[i]);
    e.l(fmt("st.param.b32 [%s], %s", pn[i], pv[i].c_str()));
  }
  e.l("call.uni rtl_vshift, (vs_op, vs_nd, vs_rem, vs_nwa, vs_kind, vs_ab, vs_a0, vs_s, vs_lim, vs_fill, vs_db, vs_top)");
  e.s += "\t}\n";
  for (uint32_t i = 0; i < nd; i++) opaque_write(e, SP_W, w.d + 32 * i);
}

// rtl_vshift: SHL / SHRL / SHRA of a wide value by a variable amount on the
// vector layout (the callee of emit_vshift; operand and destination are
// absolute shared addresses of their lane-0 word 0).
const char *kVShiftPtx = R"PTX(
.func rtl_vshift(.param .b32 vs_op, .param .b32 vs_nd, .param .b32 vs_rem, .param .b32 vs_nwa,
                 .param .b32 vs_kind, .param .b32 vs_ab, .param .b32 vs_a0, .param .b32 vs_s,
                 .param .b32 vs_lim, .param .b32 vs_fill, .param .b32 vs_db, .param .b32 vs_top)
{
  .reg .b32 %op, %nd, %rem, %nwa, %kind, %ab, %a0, %s, %lim, %fill, %db, %top, %lane;
  .reg .b32 %i, %q, %k, %jlo, %jhi, %j, %v, %x0, %x1, %r, %g, %jj, %gs, %st, %ad, %oob, %m, %nf;
  .reg .pred %pshl, %pbig, %pv, %pf, %pk1, %pk2, %pz, %pl, %ptop, %psra;
  ld.param.b32 %op, [vs_op];   ld.param.b32 %nd, [vs_nd];   ld.param.b32 %rem, [vs_rem];
  ld.param.b32 %nwa, [vs_nwa]; ld.param.b32 %kind, [vs_kind]; ld.param.b32 %ab, [vs_ab];
  ld.param.b32 %a0, [vs_a0];   ld.param.b32 %s, [vs_s];     ld.param.b32 %lim, [vs_lim];
  ld.param.b32 %fill, [vs_fill]; ld.param.b32 %db, [vs_db]; ld.param.b32 %top, [vs_top];
  mov.u32 %lane, %laneid;
  setp.eq.u32 %pshl, %op, 22;
  setp.eq.u32 %psra, %op, 24;
  selp.u32 %oob, %fill, 0, %psra;
  setp.ge.u32 %pbig, %s, %lim;
  min.u32 %s, %s, %lim;
  shr.u32 %q, %s, 5;
  and.b32 %k, %s, 31;
  setp.eq.u32 %pk1, %kind, 1;
  setp.eq.u32 %pk2, %kind, 2;
  shr.u32 %nf, %nwa, 2;
  mov.u32 %i, 0;
$VS_LOOP:
  @%pshl sub.u32 %jhi, %i, %q;
  @%pshl sub.u32 %jlo, %jhi, 1;
  @!%pshl add.u32 %jlo, %q, %i;
  @!%pshl add.u32 %jhi, %jlo, 1;
  // X(jlo) -> %x0, X(jhi) -> %x1
  mov.u32 %j, %jlo;
  bra.uni $VS_X;
$VS_X0:
  mov.u32 %x0, %v;
  mov.u32 %j, %jhi;
  bra.uni $VS_X;
$VS_X1:
  mov.u32 %x1, %v;
  @%pshl shf.l.clamp.b32 %r, %x0, %x1, %k;
  @!%pshl shf.r.clamp.b32 %r, %x0, %x1, %k;
  selp.u32 %r, %oob, %r, %pbig;
  add.u32 %m, %i, 1;
  setp.eq.u32 %ptop, %m, %nd;
  setp.ne.u32 %pz, %rem, 0;
  and.pred %ptop, %ptop, %pz;
  @%ptop shl.b32 %m, 1, %rem;
  @%ptop add.u32 %m, %m, -1;
  @%ptop and.b32 %r, %r, %m;
  // dest word i: group i / 4 of size min(4, nd - 4 g)
  shr.u32 %g, %i, 2;
  and.b32 %jj, %i, 3;
  shl.b32 %gs, %g, 2;
  sub.u32 %gs, %nd, %gs;
  min.u32 %gs, %gs, 4;
  shl.b32 %st, %gs, 2;
  mad.lo.u32 %ad, %st, %lane, %db;
  mad.lo.u32 %ad, %g, 512, %ad;
  mad.lo.u32 %ad, %jj, 4, %ad;
  st.shared.u32 [%ad], %r;
  add.u32 %i, %i, 1;
  setp.lt.u32 %pl, %i, %nd;
  @%pl bra.uni $VS_LOOP;
  ret;
$VS_X:
  // word %j of the operand (extended): 0 / sign fill beyond nwa
  setp.lt.u32 %pv, %j, %nwa;
  mov.u32 %v, %oob;
  @%pk1 mad.lo.u32 %ad, %j, 4, %ab;
  @%pk1 bra.uni $VS_LD;
  @%pk2 bra.uni $VS_VEC;
  setp.eq.u32 %pz, %j, 0;
  @%pz mov.u32 %v, %a0;
  bra.uni $VS_RET;
$VS_VEC:
  shr.u32 %g, %j, 2;
  and.b32 %jj, %j, 3;
  setp.lt.u32 %pf, %g, %nf;
  shl.b32 %gs, %g, 2;
  sub.u32 %gs, %nwa, %gs;
  min.u32 %gs, %gs, 4;
  selp.u32 %st, 16, 0, %pf;
  @!%pf shl.b32 %st, %gs, 2;
  mad.lo.u32 %ad, %st, %lane, %ab;
  mad.lo.u32 %ad, %g, 512, %ad;
  mad.lo.u32 %ad, %jj, 4, %ad;
$VS_LD:
  @%pv ld.shared.u32 %v, [%ad];
  // SHRA: the operand's top word is read sign-extended
  add.u32 %m, %j, 1;
  setp.eq.u32 %pz, %m, %nwa;
  and.pred %pz, %pz, %psra;
  @%pz mov.u32 %v, %top;
$VS_RET:
  setp.eq.u32 %pz, %j, %jlo;
  @%pz bra.uni $VS_X0;
  bra.uni $VS_X1;
}
)PTX";

void emit_wide(Em &e, const WideRec &w, uint32_t idx) {
  const uint32_t op = w.op, wd = w.wd, nd = nwords(wd);
  WOp A, B, C;
  A.off = w.a; A.w = w.wa; A.lay = w.lays & 0xFFu;
  B.off = w.b; B.w = w.wb; B.lay = (w.lays >> 8) & 0xFFu;
  C.off = w.c; C.w = w.wc; C.lay = (w.lays >> 16) & 0xFFu;
  if (wd <= 32) begin_value(e, layout_space(value_layout(wd, false)), w.d, 1);
  else begin_value(e, SP_W, w.d, nd);
  if (op == RTLSIM_OP_MEMRD) {   // ARRSEL read of a wide entry (reading 12)
    std::string idx = reg_of(e, wword(e, A, 0, false));
    for (uint32_t i = 0; i < nd; i++) wstore(e, w.d, wd, i, emit_mem_read(e, idx, w.imm, i));
    return;
  }
  auto bin = [&](const char *ins) {
    for (uint32_t i = 0; i < nd; i++) {
      std::string xa = reg_of(e, wword(e, A, i, false)), xb = reg_of(e, wword(e, B, i, false)), r = e.R();
      e.l(fmt("%s %s, %s, %s", ins, r.c_str(), xa.c_str(), xb.c_str()));
      wstore(e, w.d, wd, i, r);
    }
  };
  switch (op) {
    case RTLSIM_OP_COPY:
    case RTLSIM_OP_SEXT:
      for (uint32_t i = 0; i < nd; i++) wstore(e, w.d, wd, i, wword(e, A, i, op == RTLSIM_OP_SEXT));
      return;
    case RTLSIM_OP_NOT:
      for (uint32_t i = 0; i < nd; i++) {
        std::string xa = reg_of(e, wword(e, A, i, false)), r = e.R();
        e.l(fmt("not.b32 %s, %s", r.c_str(), xa.c_str()));
        wstore(e, w.d, wd, i, r);
      }
      return;
    case RTLSIM_OP_AND: bin("and.b32"); return;
    case RTLSIM_OP_OR: bin("or.b32"); return;
    case RTLSIM_OP_XOR: bin("xor.b32"); return;
    case RTLSIM_OP_ADD:
    case RTLSIM_OP_SUB:
    case RTLSIM_OP_NEG: {
      std::vector<std::string> xs(nd), ys(nd), rs(nd);
      for (uint32_t i = 0; i < nd; i++) {
        if (op == RTLSIM_OP_NEG) {
          xs[i] = "0";
          ys[i] = reg_of(e, wword(e, A, i, false));
        } else {
          xs[i] = reg_of(e, wword(e, A, i, false));
          ys[i] = reg_of(e, wword(e, B, i, false));
        }
        rs[i] = e.R();
      }
      const char *base = op == RTLSIM_OP_ADD ? "add" : "sub";
      for (uint32_t i = 0; i < nd; i++) {
        const char *cc = nd == 1 ? "" : (i == 0 ? ".cc" : (i + 1 < nd ? ".cc" : ""));
        const char *car = (i == 0) ? "" : "c";
        e.l(fmt("%s%s%s.u32 %s, %s, %s", base, car, cc, rs[i].c_str(), xs[i].c_str(), ys[i].c_str()));
      }
      for (uint32_t i = 0; i < nd; i++) wstore(e, w.d, wd, i, rs[i]);
      return;
    }
    case RTLSIM_OP_MUL:
    case RTLSIM_OP_DIVU:
    case RTLSIM_OP_MODU: {
      std::string a64 = e.RD(), b64 = e.RD(), r64 = e.RD();
      std::string a0 = reg_of(e, wword(e, A, 0, false)), a1 = reg_of(e, wword(e, A, 1, false));
      std::string b0 = reg_of(e, wword(e, B, 0, false)), b1 = reg_of(e, wword(e, B, 1, false));
      e.l(fmt("mov.b64 %s, {%s, %s}", a64.c_str(), a0.c_str(), a1.c_str()));
      e.l(fmt("mov.b64 %s, {%s, %s}", b64.c_str(), b0.c_str(), b1.c_str()));
      if (op == RTLSIM_OP_MUL) {
        e.l(fmt("mul.lo.u64 %s, %s, %s", r64.c_str(), a64.c_str(), b64.c_str()));
      } else {   // b == 0 gives 0
        std::string m = e.R(), m64 = e.RD(), t = e.RD();
        e.l(fmt("set.ne.u32.u64 %s, %s, 0", m.c_str(), b64.c_str()));
        e.l(fmt("mov.b64 %s, {%s, %s}", m64.c_str(), m.c_str(), m.c_str()));
        e.l(fmt("%s.u64 %s, %s, %s", op == RTLSIM_OP_DIVU ? "div" : "rem", t.c_str(), a64.c_str(), b64.c_str()));
        e.l(fmt("and.b64 %s, %s, %s", r64.c_str(), t.c_str(), m64.c_str()));
      }
      std::string lo = e.R(), hi = e.R();
      e.l(fmt("mov.b64 {%s, %s}, %s", lo.c_str(), hi.c_str(), r64.c_str()));
      wstore(e, w.d, wd, 0, lo);
      if (nd > 1) wstore(e, w.d, wd, 1, hi);
      return;
    }
    case RTLSIM_OP_EQ: case RTLSIM_OP_NE: case RTLSIM_OP_LTU: case RTLSIM_OP_LEU: case RTLSIM_OP_GTU:
    case RTLSIM_OP_GEU: case RTLSIM_OP_LTS: case RTLSIM_OP_LES: case RTLSIM_OP_GTS: case RTLSIM_OP_GES: {
      const bool sg = op >= RTLSIM_OP_LTS;
      const uint32_t n = nwords(std::max<uint32_t>(w.wa, w.wb));
      // lexicographic compare from the least significant word up, as masks:
      // LT_i = lt_i | (eq_i & LT_{i-1}), EQ_i = eq_i & EQ_{i-1}
      std::string LT, EQ;
      for (uint32_t i = 0; i < n; i++) {
        std::string xa = reg_of(e, wword(e, A, i, sg)), xb = reg_of(e, wword(e, B, i, sg));
        std::string lt = e.R(), eq = e.R();
        const bool top_signed = sg && i == n - 1;
        e.l(fmt("set.lt.u32.%s %s, %s, %s", top_signed ? "s32" : "u32", lt.c_str(), xa.c_str(), xb.c_str()));
        e.l(fmt("set.eq.u32.u32 %s, %s, %s", eq.c_str(), xa.c_str(), xb.c_str()));
        if (i == 0) {
          LT = lt;
          EQ = eq;
        } else {
          std::string LT2 = e.R(), EQ2 = e.R();
          e.l(fmt("lop3.b32 %s, %s, %s, %s, 0xf8", LT2.c_str(), lt.c_str(), eq.c_str(), LT.c_str()));
          e.l(fmt("and.b32 %s, %s, %s", EQ2.c_str(), eq.c_str(), EQ.c_str()));
          LT = LT2;
          EQ = EQ2;
        }
      }
      std::string res = e.R();
      switch (op) {
        case RTLSIM_OP_EQ: e.l(fmt("mov.u32 %s, %s", res.c_str(), EQ.c_str())); break;
        case RTLSIM_OP_NE: e.l(fmt("not.b32 %s, %s", res.c_str(), EQ.c_str())); break;
        case RTLSIM_OP_LTU: case RTLSIM_OP_LTS: e.l(fmt("mov.u32 %s, %s", res.c_str(), LT.c_str())); break;
        case RTLSIM_OP_LEU: case RTLSIM_OP_LES: e.l(fmt("or.b32 %s, %s, %s", res.c_str(), LT.c_str(), EQ.c_str())); break;
        case RTLSIM_OP_GTU: case RTLSIM_OP_GTS: e.l(fmt("lop3.b32 %s, %s, %s, 0, 0x03", res.c_str(), LT.c_str(), EQ.c_str())); break;
        default: e.l(fmt("not.b32 %s, %s", res.c_str(), LT.c_str())); break;
      }
      std::string r = e.R();
      e.l(fmt("and.b32 %s, %s, 1", r.c_str(), res.c_str()));
      for (uint32_t i = 0; i < nd; i++) wstore(e, w.d, wd, i, i == 0 ? r : std::string("0"));
      return;
    }
    case RTLSIM_OP_MUX: {
      std::string acc;
      for (uint32_t i = 0; i < nwords(w.wa); i++) {
        std::string xa = reg_of(e, wword(e, A, i, false));
        if (acc.empty()) {
          acc = xa;
        } else {
          std::string t = e.R();
          e.l(fmt("or.b32 %s, %s, %s", t.c_str(), acc.c_str(), xa.c_str()));
          acc = t;
        }
      }
      std::string m = e.R();
      e.l(fmt("set.ne.u32.u32 %s, %s, 0", m.c_str(), acc.c_str()));
      for (uint32_t i = 0; i < nd; i++) {
        std::string tb = reg_of(e, wword(e, B, i, false)), tc = reg_of(e, wword(e, C, i, false)), r = e.R();
        e.l(fmt("lop3.b32 %s, %s, %s, %s, 0xca", r.c_str(), m.c_str(), tb.c_str(), tc.c_str()));
        wstore(e, w.d, wd, i, r);
      }
      return;
    }
    case RTLSIM_OP_CONCAT: {   // (a << wb) | b
      const uint32_t ws = w.wb >> 5, bs = w.wb & 31u;
      for (uint32_t i = 0; i < nd; i++) {
        std::string v = reg_of(e, wword(e, B, i, false));
        if (i >= ws) {
          std::string lo = reg_of(e, wword(e, A, i - ws, false)), t = e.R();
          if (bs == 0) {
            e.l(fmt("or.b32 %s, %s, %s", t.c_str(), v.c_str(), lo.c_str()));
          } else {
            std::string hi_part = e.R();
            e.l(fmt("shl.b32 %s, %s, %u", hi_part.c_str(), lo.c_str(), bs));
            std::string t2 = e.R();
            e.l(fmt("or.b32 %s, %s, %s", t2.c_str(), v.c_str(), hi_part.c_str()));
            if (i > ws) {
              std::string prev = reg_of(e, wword(e, A, i - ws - 1, false)), sh = e.R();
              e.l(fmt("shr.u32 %s, %s, %u", sh.c_str(), prev.c_str(), 32 - bs));
              e.l(fmt("or.b32 %s, %s, %s", t.c_str(), t2.c_str(), sh.c_str()));
            } else {
              e.l(fmt("mov.u32 %s, %s", t.c_str(), t2.c_str()));
            }
          }
          v = t;
        }
        wstore(e, w.d, wd, i, v);
      }
      return;
    }
    case RTLSIM_OP_SLICE: {
      const uint32_t ws = w.imm >> 5, bs = w.imm & 31u;
      for (uint32_t i = 0; i < nd; i++) {
        std::string lo = reg_of(e, wword(e, A, i + ws, false));
        if (bs == 0) {
          wstore(e, w.d, wd, i, lo);
        } else {
          std::string hi = reg_of(e, wword(e, A, i + ws + 1, false)), r = e.R();
          e.l(fmt("shf.r.clamp.b32 %s, %s, %s, %u", r.c_str(), lo.c_str(), hi.c_str(), bs));
          wstore(e, w.d, wd, i, r);
        }
      }
      return;
    }
    case RTLSIM_OP_REDAND:
    case RTLSIM_OP_REDOR:
    case RTLSIM_OP_REDXOR: {
      const uint32_t n = nwords(w.wa), rem = w.wa & 31u;
      std::string acc;
      for (uint32_t i = 0; i < n; i++) {
        std::string xa = reg_of(e, wword(e, A, i, false)), t = e.R();
        if (op == RTLSIM_OP_REDAND) {   // compare against the all-ones word of this position
          std::string m = e.R();
          e.l(fmt("set.eq.u32.u32 %s, %s, %u", m.c_str(), xa.c_str(), (i == n - 1 && rem) ? mask_of(rem) : 0xFFFFFFFFu));
          e.l(fmt("and.b32 %s, %s, 1", t.c_str(), m.c_str()));
          if (!acc.empty()) {
            std::string u = e.R();
            e.l(fmt("and.b32 %s, %s, %s", u.c_str(), acc.c_str(), t.c_str()));
            t = u;
          }
        } else if (op == RTLSIM_OP_REDOR) {
          if (acc.empty()) {
            e.l(fmt("mov.u32 %s, %s", t.c_str(), xa.c_str()));
          } else {
            e.l(fmt("or.b32 %s, %s, %s", t.c_str(), acc.c_str(), xa.c_str()));
          }
        } else {
          e.l(fmt("popc.b32 %s, %s", t.c_str(), xa.c_str()));
          if (!acc.empty()) {
            std::string u = e.R();
            e.l(fmt("add.u32 %s, %s, %s", u.c_str(), acc.c_str(), t.c_str()));
            t = u;
          }
        }
        acc = t;
      }
      std::string r = e.R();
      if (op == RTLSIM_OP_REDAND) {
        e.l(fmt("mov.u32 %s, %s", r.c_str(), acc.c_str()));
      } else if (op == RTLSIM_OP_REDOR) {
        std::string m = e.R();
        e.l(fmt("set.ne.u32.u32 %s, %s, 0", m.c_str(), acc.c_str()));
        e.l(fmt("and.b32 %s, %s, 1", r.c_str(), m.c_str()));
      } else {
        e.l(fmt("and.b32 %s, %s, 1", r.c_str(), acc.c_str()));
      }
      for (uint32_t i = 0; i < nd; i++) wstore(e, w.d, wd, i, i == 0 ? r : std::string("0"));
      return;
    }
    default:   // SHL / SHRL / SHRA by a variable amount
      if (jit_vwide()) emit_vshift(e, w, A, B);
      else generic_wide(e, w, idx);   // the interpreter's generic path (row layout)
      return;
  }
}

// ----------------------------------------------------------- loads / stores --
const char *kArenaTag[4] = {"c", "n", "x", "i"};   // cur, nxt, xnet, in

// (r2) source address of a cp.async: LDGSTS has only a ~2 KB immediate on
// the global side, so an [window + immediate] address costs IADD3 + IMAD.X
// per row anyway; one IMAD.WIDE (row x stride + base) is shorter and keeps
// no window register live
// (measured config 4 TMEM: 55.3 ms/cycle with windows vs 55.9 with IMAD.WIDE:
// windows stay the default, RTLSIM_JIT_LDMAD=1 for A/B)
std::string ldaddr(Em &e, const char *sreg, uint32_t row, const char *base) {
  if (!e.nspec || !getenv("RTLSIM_JIT_LDMAD")) return gaddr(e, sreg, row, base);
  std::string a = e.RD();
  e.l(fmt("mad.wide.u32 %s, %%%s, %u, %%%s", a.c_str(), sreg, row, base));
  return a;
}
// (r2, RTLSIM_JIT_LD16=1, default off: config 4 TMEM 55.8 vs 55.3 ms/cycle —
// 40 % fewer LDGSTS but two more live registers and more spills)
bool jit_ld16() {
  const char *e = getenv("RTLSIM_JIT_LD16");
  return e ? atoi(e) != 0 : false;
}

void emit_ld(Em &e, uint32_t arena, uint32_t cls, uint32_t row, uint32_t slot, uint32_t nw) {
  const char *A = kArenaTag[arena];
  std::string addr;
  if (cls == CLS_U32 && nw >= 2 && jit_ld16() && !jit_vwide() && !e.compact) {
    // (r2) a wide register's nw consecutive rows, four per 16-byte cp.async:
    // lane l copies bytes 16 (l & 7) .. +15 of row r0 + (l >> 3) of the tile
    // into word row (l >> 3) of the slot (%vsm, %vdl: the per-lane offsets)
    e.used_v = true;
    begin_value(e, SP_W, slot, nw, true);
    std::string tb = e.RD();
    e.l(fmt("add.s64 %s, %%tb_%s3, %%vdl", tb.c_str(), A));
    for (uint32_t g = 0; g < nw; g += 4) {
      std::string a = e.RD();
      e.l(fmt("mad.wide.u32 %s, %%N4, %u, %s", a.c_str(), row + g, tb.c_str()));
      const uint32_t k = std::min<uint32_t>(4u, nw - g);
      const char *pr = k == 1 ? "@%pl8 " : k == 2 ? "@%pl16 " : k == 3 ? "@%pl24 " : "";
      e.l(fmt("%scp.async.cg.shared.global [%%vsm+%u], [%s], 16", pr, (slot + 32u * g) * 4u, a.c_str()));
    }
    for (uint32_t i = 0; i < nw; i++) opaque_write(e, SP_W, slot + 32 * i);
    return;
  }
  switch (cls) {
    case CLS_U32:
      begin_value(e, SP_W, slot, nw, true);
      for (uint32_t i = 0; i < nw; i++) {
        std::string ai = ldaddr(e, "N4", row + i, fmt("tb_%s3", A).c_str());
        if (nw >= 2 && jit_vwide())   // into the word's place in its group
          e.l(fmt("cp.async.ca.shared.global [%s+%u], [%s], 4", kLaneBase[vgs(nw, i / 4u)], vbyte(e, slot, nw, i),
                  ai.c_str()));
        else
          e.l(fmt("cp.async.ca.shared.global [%%rw+%u], [%s], 4", xoff(e, SP_W, slot + 32 * i) * 4, ai.c_str()));
        opaque_write(e, SP_W, slot + 32 * i);
      }
      break;
    case CLS_U16:
      begin_value(e, SP_H, slot, 1, true);
      addr = ldaddr(e, "N2", row, fmt("tb_%s2", A).c_str());
      e.l(fmt("@%%pl16 cp.async.ca.shared.global [%%rw+%u], [%s], 4", xoff(e, SP_H, slot) * 4, addr.c_str()));
      opaque_write(e, SP_H, slot);
      break;
    case CLS_U8:
      begin_value(e, SP_B, slot, 1, true);
      addr = ldaddr(e, "N", row, fmt("tb_%s1", A).c_str());
      e.l(fmt("@%%pl8 cp.async.ca.shared.global [%%rw+%u], [%s], 4", xoff(e, SP_B, slot) * 4, addr.c_str()));
      opaque_write(e, SP_B, slot);
      break;
    default:
      begin_value(e, SP_S, slot, 1, true);
      addr = ldaddr(e, "Nb", row, fmt("tb_%s0", A).c_str());
      e.l(fmt("@%%pl0 cp.async.ca.shared.global [%%smb+%u], [%s], 4", xoff(e, SP_S, slot) * 4, addr.c_str()));
      opaque_write(e, SP_S, slot);
      break;
  }
}

void emit_dig(Em &e, uint32_t key, const std::string &v) {
  if (!e.dig) return;
  std::string skip = e.L("nd");
  e.l(fmt("@!%%pdig bra.uni %s", skip.c_str()));
  e.s += "\t{\n\t.param .b64 dp0;\n\t.param .b32 dp1;\n\t.param .b32 dp2;\n";
  e.l("st.param.b64 [dp0], %dig");
  e.l(fmt("st.param.b32 [dp1], %u", key));
  e.l(fmt("st.param.b32 [dp2], %s", v.c_str()));
  e.l("call.uni rtl_dig, (dp0, dp1, dp2)");
  e.s += "\t}\n";
  e.lab(skip);
}

void emit_st(Em &e, uint32_t code, uint32_t cls, uint32_t nw, uint32_t lay, uint32_t slot, uint32_t row,
             uint32_t aux) {
  const bool dg = code == CODE_ST_REG;
  auto u32word = [&](uint32_t i) {   // word i of a U32-layout source of nw words
    return (nw >= 2 && jit_vwide()) ? vword(e, slot, nw, i) : lds(e, SP_W, slot + 32 * i);
  };
  if (code == CODE_ST_PORT) {   // write-port words of this cycle (applied after the cycle)
    for (uint32_t i = 0; i < nw; i++) {
      std::string v = lay == LC_U32 ? u32word(i) : fetch_narrow(e, lay, slot, 32);
      std::string addr = gaddr(e, "N4", row + i, "portb");
      e.l(fmt("st.global.u32 [%s], %s", addr.c_str(), v.c_str()));
    }
    return;
  }
  if (code == CODE_ST_OUT) {
    for (uint32_t i = 0; i < nw; i++) {
      std::string v;
      if (lay == LC_U32) {
        v = u32word(i);
      } else {
        v = fetch_narrow(e, lay, slot, 32);
      }
      std::string addr = gaddr(e, "N4", row + i, "outb");
      e.l(fmt("st.global.u32 [%s], %s", addr.c_str(), v.c_str()));
      emit_dig(e, row + i + 1, v);
    }
    return;
  }
  const char *A = code == CODE_ST_REG ? "n" : "x";
  std::string addr;
  switch (cls) {
    case CLS_U32:
      for (uint32_t i = 0; i < nw; i++) {
        std::string v = u32word(i);
        std::string ai = gaddr(e, "N4", row + i, fmt("tb_%s3", A).c_str());
        e.l(fmt("st.global.u32 [%s], %s", ai.c_str(), v.c_str()));
        if (dg) emit_dig(e, aux + i + 1u + 0x80000000u, v);
      }
      return;
    case CLS_U16:
    case CLS_U8: {
      // 32 byte / half-word lanes: 8 or 16 lanes copy the packed words
      std::string t = e.R();
      const char *pl = cls == CLS_U8 ? "%pl8" : "%pl16";
      e.l(fmt("@%s ld.shared.u32 %s, [%%rw+%u]", pl, t.c_str(), xoff(e, cls == CLS_U8 ? SP_B : SP_H, slot) * 4));
      note_read(e, cls == CLS_U8 ? SP_B : SP_H, slot);
      note_read(e, layout_space(lay), slot);
      addr = cls == CLS_U8 ? gaddr(e, "N", row, fmt("tb_%s1", A).c_str()) : gaddr(e, "N2", row, fmt("tb_%s2", A).c_str());
      e.l(fmt("@%s st.global.u32 [%s], %s", pl, addr.c_str(), t.c_str()));
      if (dg && e.dig) emit_dig(e, aux + 1u + 0x80000000u, fetch_narrow(e, lay, slot, 16));
      return;
    }
    default: {
      std::string t = lds(e, SP_S, slot);
      addr = gaddr(e, "Nb", row, fmt("tb_%s0", A).c_str());
      e.l(fmt("@%%pl0 st.global.u32 [%s], %s", addr.c_str(), t.c_str()));
      if (dg && e.dig) {
        std::string b = e.R(), b2 = e.R();
        e.l(fmt("shr.b32 %s, %s, %%lane", b.c_str(), t.c_str()));
        e.l(fmt("and.b32 %s, %s, 1", b2.c_str(), b.c_str()));
        emit_dig(e, aux + 1u + 0x80000000u, b2);
      }
      return;
    }
  }
}

// register store with the width conversion folded in (CODE_ST_REGC):
// q <- d mod 2^w_q, d read from its own slot (layout slay, width sw)
void emit_st_conv(Em &e, uint32_t tcls, uint32_t tnw, uint32_t slay, uint32_t sw, uint32_t slot, uint32_t row,
                  uint32_t tw, uint32_t aux) {
  WOp S;
  S.off = slot;
  S.w = sw;
  S.lay = slay;
  auto word = [&](uint32_t i) { return reg_of(e, wword(e, S, i, false)); };
  auto masked = [&](const std::string &v, uint32_t bits) {
    if (bits >= 32) return v;
    std::string m = e.R();
    e.l(fmt("and.b32 %s, %s, %u", m.c_str(), v.c_str(), mask_of(bits)));
    return m;
  };
  switch (tcls) {
    case CLS_U32:
      for (uint32_t i = 0; i < tnw; i++) {
        std::string v = word(i);
        if (i == tnw - 1 && (tw & 31u)) v = masked(v, tw & 31u);
        std::string ai = gaddr(e, "N4", row + i, "tb_n3");
        e.l(fmt("st.global.u32 [%s], %s", ai.c_str(), v.c_str()));
        emit_dig(e, aux + i + 1u + 0x80000000u, v);
      }
      return;
    case CLS_U16:
    case CLS_U8: {   // one byte / half-word per lane, 32 / 64 contiguous bytes
      std::string v = masked(word(0), tw), ai;
      if (tcls == CLS_U8) {
        ai = gaddr(e, "N", row, "tbb1");
        e.l(fmt("st.global.u8 [%s], %s", ai.c_str(), v.c_str()));
      } else {
        ai = gaddr(e, "N2", row, "tbb2");
        e.l(fmt("st.global.u16 [%s], %s", ai.c_str(), v.c_str()));
      }
      emit_dig(e, aux + 1u + 0x80000000u, v);
      return;
    }
    default: {   // 1-bit register: bit 0 of the source, packed by ballot
      std::string v = word(0), p = e.P(), m = e.R();
      e.l(fmt("setp.ne.u32 %s, %s, 0", p.c_str(), masked(v, 1).c_str()));
      e.l(fmt("vote.sync.ballot.b32 %s, %s, 0xffffffff", m.c_str(), p.c_str()));
      std::string ai = gaddr(e, "Nb", row, "tb_n0");
      e.l(fmt("@%%pl0 st.global.u32 [%s], %s", ai.c_str(), m.c_str()));
      if (e.dig) {
        std::string b = e.R();
        e.l(fmt("selp.u32 %s, 1, 0, %s", b.c_str(), p.c_str()));
        emit_dig(e, aux + 1u + 0x80000000u, b);
      }
      return;
    }
  }
}

void emit_ld_const(Em &e, const Program &G, uint32_t slot, uint32_t pool, uint32_t nw, bool bcast) {
  begin_value(e, bcast ? SP_S : SP_W, slot, nw);
  for (uint32_t i = 0; i < nw; i++) {
    std::string v = e.R();
    e.l(fmt("mov.u32 %s, %u", v.c_str(), G.const_pool[pool + i]));
    if (bcast) sts(e, SP_S, slot + i, v);
    else sts(e, SP_W, slot + 32 * i, v);
  }
}

// convert program.h truth-table order (bit k = f(a=k&1, b=k>>1&1, c=k>>2)) to
// PTX lop3 order (bit j = f(a=j>>2&1, b=j>>1&1, c=j&1))
uint32_t lop3_lut(uint32_t lut) {
  uint32_t r = 0;
  for (uint32_t j = 0; j < 8; j++) {
    const uint32_t a = (j >> 2) & 1u, b = (j >> 1) & 1u, c = j & 1u;
    r |= ((lut >> (a | (b << 1) | (c << 2))) & 1u) << j;
  }
  return r;
}

void emit_bit(Em &e, const BitDesc &q) {
  const uint32_t lut = q.x & 0xFFu, immf = q.x >> 8;
  const uint32_t f[3] = {q.y >> 16, q.z & 0xFFFFu, q.z >> 16};
  begin_value(e, SP_S, q.y & 0xFFFFu, 1);
  std::string v[3];
  for (int k = 0; k < 3; k++) {
    v[k] = e.R();
    // an input the truth table ignores (unary / binary ops) is not read: a
    // load of its placeholder slot would race with the slot's real writers
    bool used = false;
    for (uint32_t idx = 0; idx < 8; idx++)
      used |= ((lut >> idx) & 1u) != ((lut >> (idx ^ (1u << k))) & 1u);
    if (!used) e.l(fmt("mov.u32 %s, 0", v[k].c_str()));
    else if (immf & (1u << k)) e.l(fmt("mov.u32 %s, %u", v[k].c_str(), (f[k] & 1u) ? 0xFFFFFFFFu : 0u));
    else v[k] = lds(e, SP_S, f[k]);
  }
  std::string r = e.R();
  e.l(fmt("lop3.b32 %s, %s, %s, %s, 0x%02x", r.c_str(), v[0].c_str(), v[1].c_str(), v[2].c_str(), lop3_lut(lut)));
  sts(e, SP_S, q.y & 0xFFFFu, r);
}

// Lane-parallel bit ops (RTLSIM_JIT_BITBATCH=k, default 0 = off): the 1-bit
// ops of one warp's step that share one truth table (immediates folded in),
// in groups of >= k; lane i evaluates op i of the group on the packed words
// (32 stimuli each), its four operand / result slot addresses read from a
// per-partition table (one LDG.128 per lane): up to 32 ops in ~11 warp
// instructions instead of ~4-5 each (every lane computing the same word).
// Measured off by default: config 3 steps hold ~28 bit ops over 4 warps and
// ~6 truth tables, so groups average 3.3 ops, and batched results can no
// longer be forwarded in registers (total SASS +2 %).
uint32_t jit_bitbatch() {
  const char *e = getenv("RTLSIM_JIT_BITBATCH");
  return e ? (uint32_t)atoi(e) : 0u;
}
// truth table with the immediate operands substituted (they become unused)
uint32_t bit_fold_lut(const BitDesc &q) {
  uint32_t lut = q.x & 0xFFu;
  const uint32_t immf = q.x >> 8;
  const uint32_t f[3] = {q.y >> 16, q.z & 0xFFFFu, q.z >> 16};
  for (uint32_t k = 0; k < 3; k++) {
    if (!(immf & (1u << k))) continue;
    uint32_t n = 0;
    for (uint32_t j = 0; j < 8; j++) {
      const uint32_t src = (j & ~(1u << k)) | ((f[k] & 1u) << k);
      n |= ((lut >> src) & 1u) << j;
    }
    lut = n;
  }
  return lut;
}
bool lut_uses(uint32_t lut, uint32_t k) {
  for (uint32_t idx = 0; idx < 8; idx++)
    if (((lut >> idx) & 1u) != ((lut >> (idx ^ (1u << k))) & 1u)) return true;
  return false;
}
void emit_bit_batch(Em &e, const std::vector<BitDesc> &ops, uint32_t lut) {
  const uint32_t n = (uint32_t)ops.size();
  for (const BitDesc &q : ops) begin_value(e, SP_S, q.y & 0xFFFFu, 1, true);
  const uint32_t base = e.bittab ? (uint32_t)(e.bittab->size() / 4) : 0;
  for (const BitDesc &q : ops) {
    const uint32_t d = q.y & 0xFFFFu;
    const uint32_t f[3] = {q.y >> 16, q.z & 0xFFFFu, q.z >> 16};
    uint32_t ent[4];
    for (uint32_t k = 0; k < 3; k++) {
      if (lut_uses(lut, k)) {
        note_read(e, SP_S, f[k]);
        ent[k] = xoff(e, SP_S, f[k]) * 4;
      } else {
        ent[k] = xoff(e, SP_S, d) * 4;   // ignored input: the lane's own result word
      }
    }
    ent[3] = xoff(e, SP_S, d) * 4;
    if (e.bittab && !e.dry) e.bittab->insert(e.bittab->end(), ent, ent + 4);
  }
  std::string p = e.P(), t[4], a[4], v[3], r = e.R();
  for (int k = 0; k < 4; k++) { t[k] = e.R(); a[k] = e.R(); }
  for (int k = 0; k < 3; k++) v[k] = e.R();
  e.l(fmt("setp.lt.u32 %s, %%lane, %u", p.c_str(), n));
  e.l(fmt("@%s ld.global.nc.v4.u32 {%s, %s, %s, %s}, [%%bitl+%u]", p.c_str(), t[0].c_str(), t[1].c_str(),
          t[2].c_str(), t[3].c_str(), base * 16));
  for (int k = 0; k < 4; k++) e.l(fmt("add.u32 %s, %s, %%smb", a[k].c_str(), t[k].c_str()));
  for (int k = 0; k < 3; k++) e.l(fmt("@%s ld.shared.u32 %s, [%s]", p.c_str(), v[k].c_str(), a[k].c_str()));
  e.l(fmt("lop3.b32 %s, %s, %s, %s, 0x%02x", r.c_str(), v[0].c_str(), v[1].c_str(), v[2].c_str(), lop3_lut(lut)));
  e.l(fmt("@%s st.shared.u32 [%s], %s", p.c_str(), a[3].c_str(), r.c_str()));
  for (const BitDesc &q : ops) opaque_write(e, SP_S, q.y & 0xFFFFu);
}

// (r2) Lane-parallel bit ops with a truth table per lane (RTLSIM_JIT_BITANY=k,
// default 0 = off: config 4 TMEM 59.1 ms/cycle with k = 8 vs 55.4 without —
// 3 % less code, but the table load sits on every step's critical path): the step's 1-bit ops are dealt to the warps in chunks
// of up to 32 (chunk c to op-lane c mod L) instead of one by one; lane i of
// the chunk evaluates op i — operand / result offsets and its own truth table
// (immediates folded in) from one LDG.128 of a per-partition table — as the
// OR of the minterms its table selects: one LOP3 per minterm any op of the
// chunk uses, masked by a BFE of the lane's table bit where the ops differ.
// A chunk of n ops costs ~12-30 warp instructions instead of ~5 n (every lane
// computing the same packed word, one op after another); chunks smaller
// than k keep the per-op code. The JIT is instruction-fetch bound
// (DESIGN.md §5.2b), so the total code is what counts.
uint32_t jit_bitany() {
  const char *e = getenv("RTLSIM_JIT_BITANY");
  return e ? (uint32_t)atoi(e) : 0u;
}
// the bit ops warp w evaluates in step s (indices into G.bitdesc), in chunks
void warp_bits(const Program &G, uint32_t s, uint32_t w, std::vector<std::vector<uint32_t>> &out) {
  out.clear();
  const uint32_t b0 = G.bit_ptr[s], b1 = G.bit_ptr[s + 1], n = b1 - b0, k = jit_bitany();
  if (k && n >= k && jit_split() == 0 && jit_bitbatch() == 0) {
    const uint32_t nch = (n + 31u) / 32u, sz = (n + nch - 1u) / nch;
    for (uint32_t c = w; c < nch; c += G.L) {
      std::vector<uint32_t> ch;
      for (uint32_t i = b0 + c * sz; i < std::min(b1, b0 + (c + 1u) * sz); i++) ch.push_back(i);
      if (!ch.empty()) out.push_back(std::move(ch));
    }
    return;
  }
  for (uint32_t i = b0 + w; i < b1; i += G.L) out.push_back({i});
}
void emit_bit_batch_any(Em &e, const Program &G, const std::vector<uint32_t> &idx) {
  const uint32_t n = (uint32_t)idx.size();
  for (uint32_t i : idx) begin_value(e, SP_S, G.bitdesc[i].y & 0xFFFFu, 1, true);
  const uint32_t base = e.bittab ? (uint32_t)(e.bittab->size() / 4) : 0;
  uint32_t any = 0, all = 0xFFu, used = 0;
  for (uint32_t i : idx) {
    const BitDesc &q = G.bitdesc[i];
    const uint32_t lut = bit_fold_lut(q), d = q.y & 0xFFFFu;
    const uint32_t f[3] = {q.y >> 16, q.z & 0xFFFFu, q.z >> 16};
    any |= lut;
    all &= lut;
    uint32_t ent[4];
    for (uint32_t k = 0; k < 3; k++) {
      if (lut_uses(lut, k)) {
        used |= 1u << k;
        note_read(e, SP_S, f[k]);
        ent[k] = xoff(e, SP_S, f[k]) * 4;
      } else {
        ent[k] = xoff(e, SP_S, d) * 4;   // ignored input: the lane's own result word
      }
    }
    ent[3] = xoff(e, SP_S, d) * 4 | (lut << 24);
    if (e.bittab && !e.dry) e.bittab->insert(e.bittab->end(), ent, ent + 4);
  }
  std::string p = e.P(), t[4], a[4], v[3], L = e.R(), dd = e.R();
  for (int k = 0; k < 4; k++) { t[k] = e.R(); a[k] = e.R(); }
  e.l(fmt("setp.lt.u32 %s, %%lane, %u", p.c_str(), n));
  e.l(fmt("@%s ld.global.nc.v4.u32 {%s, %s, %s, %s}, [%%bitl+%u]", p.c_str(), t[0].c_str(), t[1].c_str(),
          t[2].c_str(), t[3].c_str(), base * 16));
  e.l(fmt("shr.u32 %s, %s, 24", L.c_str(), t[3].c_str()));
  e.l(fmt("and.b32 %s, %s, 16777215", dd.c_str(), t[3].c_str()));
  e.l(fmt("add.u32 %s, %s, %%smb", a[3].c_str(), dd.c_str()));
  for (int k = 0; k < 3; k++) {
    v[k] = e.R();
    if (!(used & (1u << k))) {
      e.l(fmt("mov.u32 %s, 0", v[k].c_str()));   // no op of the chunk reads it
      continue;
    }
    e.l(fmt("add.u32 %s, %s, %%smb", a[k].c_str(), t[k].c_str()));
    e.l(fmt("@%s ld.shared.u32 %s, [%s]", p.c_str(), v[k].c_str(), a[k].c_str()));
  }
  std::string r;
  for (uint32_t j = 0; j < 8; j++) {
    if (!((any >> j) & 1u)) continue;
    if (j & ~used) continue;   // an input no op reads is 0 here: minterms needing it are 0
    const uint32_t mt = ((j & 1u) ? 0xF0u : 0x0Fu) & ((j & 2u) ? 0xCCu : 0x33u) & ((j & 4u) ? 0xAAu : 0x55u);
    std::string m = e.R(), nr = e.R();
    e.l(fmt("lop3.b32 %s, %s, %s, %s, 0x%02x", m.c_str(), v[0].c_str(), v[1].c_str(), v[2].c_str(), mt));
    if ((all >> j) & 1u) {
      if (r.empty()) r = m;
      else { e.l(fmt("or.b32 %s, %s, %s", nr.c_str(), r.c_str(), m.c_str())); r = nr; }
    } else {
      std::string M = e.R();
      e.l(fmt("bfe.s32 %s, %s, %u, 1", M.c_str(), L.c_str(), j));
      if (r.empty()) e.l(fmt("and.b32 %s, %s, %s", nr.c_str(), m.c_str(), M.c_str()));
      else e.l(fmt("lop3.b32 %s, %s, %s, %s, 0xf8", nr.c_str(), r.c_str(), m.c_str(), M.c_str()));   // r | (m & M)
      r = nr;
    }
  }
  if (r.empty()) {
    r = e.R();
    e.l(fmt("mov.u32 %s, 0", r.c_str()));
  }
  e.l(fmt("@%s st.shared.u32 [%s], %s", p.c_str(), a[3].c_str(), r.c_str()));
  for (uint32_t i : idx) opaque_write(e, SP_S, G.bitdesc[i].y & 0xFFFFu);
}

// RTLSIM_JIT_STATS: PTX instruction lines per descriptor kind (stderr at exit)
struct EmitStats {
  std::mutex mu;
  std::map<std::string, std::pair<uint64_t, uint64_t>> m;   // kind -> (count, lines)
  ~EmitStats() {
    if (m.empty()) return;
    for (auto &kv : m)
      fprintf(stderr, "jit-stats %-14s %9llu ops %11llu ptx lines %6.1f/op\n", kv.first.c_str(),
              (unsigned long long)kv.second.first, (unsigned long long)kv.second.second,
              (double)kv.second.second / (double)std::max<uint64_t>(kv.second.first, 1));
  }
};
EmitStats g_emit_stats;
size_t count_lines(const std::string &s, size_t from) {
  size_t n = 0;
  for (size_t i = from; i < s.size(); i++) n += s[i] == ';';
  return n;
}
void note_kind(Em &e, const std::string &kind, size_t from) {
  static const bool on = getenv("RTLSIM_JIT_STATS") != nullptr;
  if (!on || e.dry || e.probe) return;
  std::lock_guard<std::mutex> g(g_emit_stats.mu);
  auto &x = g_emit_stats.m[kind];
  x.first++;
  x.second += count_lines(e.s, from);
}

void emit_desc_(Em &e, const Program &G, const Desc &q);
void desc_keys(const Program &G, const Desc &q, std::vector<uint64_t> &src, std::vector<uint64_t> &dst, bool *ld);
// (r2) TMEM operands of a descriptor: every word not already in a register
// is loaded up front — runs of consecutive columns as vector tcgen05.ld
// (.x2 .. .x32), one tcgen05.wait::ld for all — and handed to the emitter as
// forwarded registers (lds() then finds them)
void tm_cols_of(Em &e, const Program &G, const Desc &q, std::vector<uint32_t> &cols) {
  std::vector<uint64_t> src, dst;
  bool ld = false;
  desc_keys(G, q, src, dst, &ld);
  const uint32_t code = q.x & 0xFFu;
  uint32_t lo = 0, hi = UINT32_MAX;   // SLICE of a wide operand: only the words it reads
  if (code == CODE_WIDE && G.wide[q.y].op == RTLSIM_OP_SLICE) {
    const WideRec &r = G.wide[q.y];
    lo = r.imm / 32u;
    hi = (r.imm + r.wd - 1u) / 32u;
  }
  for (uint64_t k : src) {
    const uint32_t off = (uint32_t)k;
    if ((k >> 32) != SP_W || !in_tmem(off) || !fwd_get(e, k).empty()) continue;
    if (code == CODE_WIDE && G.wide[q.y].op == RTLSIM_OP_SLICE) {
      const uint32_t i = (off - G.wide[q.y].a) / 32u;
      if (i < lo || i > hi) continue;
    }
    cols.push_back((off - kTmemBase) / 32u);
  }
}
// RTLSIM_JIT_TMGROUP=g: the TMEM operands of g consecutive descriptors of a
// warp's step are loaded together (one wait); default 1
uint32_t jit_tmgroup() {
  const char *e = getenv("RTLSIM_JIT_TMGROUP");
  return e ? std::max(1, atoi(e)) : 1u;
}
void tm_prefetch_cols(Em &e, std::vector<uint32_t> &cols);
void tm_prefetch(Em &e, const Program &G, const Desc &q) {
  std::vector<uint32_t> cols;
  tm_cols_of(e, G, q, cols);
  tm_prefetch_cols(e, cols);
}
void tm_prefetch_cols(Em &e, std::vector<uint32_t> &cols) {
  if (cols.empty()) return;
  std::sort(cols.begin(), cols.end());
  cols.erase(std::unique(cols.begin(), cols.end()), cols.end());
  std::vector<std::pair<uint32_t, std::string>> got;
  for (size_t i = 0; i < cols.size();) {
    size_t j = i + 1;
    while (j < cols.size() && cols[j] == cols[j - 1] + 1) j++;
    uint32_t c = cols[i], rem = (uint32_t)(j - i);
    while (rem) {
      uint32_t n = 1;
      while (n * 2 <= rem && n * 2 <= 32u && (c % (n * 2)) == 0) n *= 2;   // naturally aligned chunks
      std::string regs;
      for (uint32_t t = 0; t < n; t++) {
        std::string r = e.R();
        regs += (t ? ", " : "") + r;
        got.push_back({c + t, r});
      }
      e.l(fmt("tcgen05.ld.sync.aligned.32x32b.x%u.b32 {%s}, [%%tmt+%u]", n, regs.c_str(), c));
      c += n;
      rem -= n;
    }
    i = j;
  }
  e.l("tcgen05.wait::ld.sync.aligned");
  for (auto &g : got) {
    const uint32_t off = kTmemBase + 32u * g.first;
    const uint64_t k = skey(SP_W, off);
    if (e.probe) e.log->rd[k].push_back(e.step);
    inst_read(e, SP_W, off);
    e.fwd[k] = Em::Fwd{g.second, e.step - 1, e.opn};
  }
}
void emit_desc(Em &e, const Program &G, const Desc &q) {
  e.opn++;
  const size_t from = e.s.size();
  if (G.tmem_cols && !e.dry && e.fwd_max > 0) tm_prefetch(e, G, q);
  emit_desc_(e, G, q);
  if (!e.vpend.empty()) {   // every wide result stores whole groups; a partial one is a bug
    fprintf(stderr, "rtlsim jit: internal error: incomplete wide-value group store\n");
    abort();
  }
  const uint32_t code = q.x & 0xFFu;
  std::string kind = code < 32u ? "narrow" : code == CODE_WIDE ? "wide" : code == CODE_LD_CONST ? "ld_const"
                   : (code == CODE_LD_REG || code == CODE_LD_X || code == CODE_LD_IN) ? "ld"
                   : code == CODE_ST_REGC ? "st_conv" : "st";
  if (code < 32u) kind += ((q.x >> 17) & 7u) == LC_BIT ? ":bit" : "";
  if (code == CODE_WIDE && getenv("RTLSIM_JIT_STATS_WIDE")) kind += fmt(":%u", G.wide[q.y].op);
  note_kind(e, kind, from);
}
void emit_desc_(Em &e, const Program &G, const Desc &q) {
  const uint32_t code = q.x & 0xFFu;
  if (code < 32u) {
    emit_narrow(e, q);
    return;
  }
  if (code == CODE_WIDE) {
    emit_wide(e, G.wide[q.y], q.y);
    return;
  }
  const uint32_t cls = (q.x >> 8) & 3u, nw = (q.x >> 12) & 63u;
  switch (code) {
    case CODE_LD_REG: emit_ld(e, 0, cls, q.z, q.y, nw); break;
    case CODE_LD_X: emit_ld(e, 2, cls, q.z, q.y, nw); break;
    case CODE_LD_IN: emit_ld(e, 3, cls, q.z, q.y, nw); break;
    case CODE_LD_CONST: emit_ld_const(e, G, q.y, q.z, nw, ((q.x >> 18) & 1u) != 0); break;
    case CODE_ST_REG: case CODE_ST_X: case CODE_ST_OUT: case CODE_ST_PORT:
      emit_st(e, code, cls, nw, (q.x >> 18) & 7u, q.y, q.z, q.w);
      break;
    case CODE_ST_REGC:
      emit_st_conv(e, cls, nw, (q.x >> 18) & 7u, q.x >> 21, q.y, q.z & 0xFFFFFu, q.z >> 20, q.w);
      break;
    default: break;
  }
}

// forwarding distance in steps (RTLSIM_JIT_FWD; 0 disables). A first version
// let bit ops load the placeholder slot of an operand their truth table
// ignores; that racy read seeded a stale forwarded value (wrong registers in
// one config-4 partition; found by tools/bisect4.py, compute-sanitizer
// racecheck and tools/fwd_hazard_check.py, fixed in emit_bit / lds).
bool jit_dse() {
  const char *e = getenv("RTLSIM_JIT_DSE");
  return e ? atoi(e) != 0 : true;
}
int32_t jit_fwd_steps() {
  const char *e = getenv("RTLSIM_JIT_FWD");
  return e ? atoi(e) : 2;
}

std::string func_proto(const std::string &name) {
  std::string s = ".func " + name + "(";
  for (int i = 0; i < kN32; i++) s += fmt("%s.param .b32 a_%s", i ? ", " : "", kCtx32[i]);
  for (int i = 0; i < kN64; i++) s += fmt(", .param .b64 a_%s", kCtx64[i]);
  return s + ")";
}

// one step function: steps [s0, s1). The code is laid out per warp — each
// warp's ops of all the steps follow each other, with the step barrier
// (bar.sync 0, counted per CTA, not per PC) inside every warp's stream — so
// a warp's instruction fetch is sequential across steps instead of jumping
// over the other warps' code at every step.
// ---------------------------------------------- split-phase step barrier --
// slot row keys of a value (layout lay at slot offset off, width w)
void value_keys(uint32_t lay, uint32_t off, uint32_t w, std::vector<uint64_t> &out) {
  if (lay == LC_IMM || w == 0) return;
  if (lay == LC_U32) {
    for (uint32_t i = 0; i < nwords(w); i++) out.push_back(skey(SP_W, off + 32 * i));
  } else if (lay == LC_BCAST) {
    for (uint32_t i = 0; i < nwords(w); i++) out.push_back(skey(SP_S, off + i));
  } else {
    out.push_back(skey(layout_space(lay), off));
  }
}
// operand and destination slot keys of a descriptor (every operand, whether
// or not the emitter forwards it); *ld: a cp.async load
void desc_keys(const Program &G, const Desc &q, std::vector<uint64_t> &src, std::vector<uint64_t> &dst, bool *ld) {
  const uint32_t code = q.x & 0xFFu;
  *ld = false;
  if (code < 32u) {
    const uint32_t la = (q.x >> 8) & 7u, lb = (q.x >> 11) & 7u, lc = (q.x >> 14) & 7u, ldl = (q.x >> 17) & 7u;
    value_keys(la, q.y >> 16, 32, src);
    if ((q.w >> 11) & 1u) value_keys(lb, q.z & 0xFFFFu, 32, src);
    if ((q.w >> 12) & 1u) value_keys(lc, q.z >> 16, 32, src);
    value_keys(ldl, q.y & 0xFFFFu, 32, dst);
  } else if (code == CODE_WIDE) {
    const WideRec &r = G.wide[q.y];
    value_keys(r.lays & 0xFFu, r.a, r.wa, src);
    value_keys((r.lays >> 8) & 0xFFu, r.b, r.wb, src);
    value_keys((r.lays >> 16) & 0xFFu, r.c, r.wc, src);
    value_keys(r.wd <= 32 ? value_layout(r.wd, false) : LC_U32, r.d, r.wd, dst);
  } else if (code == CODE_LD_REG || code == CODE_LD_X || code == CODE_LD_IN) {
    *ld = true;
    const uint32_t cls = (q.x >> 8) & 3u, nw = (q.x >> 12) & 63u;
    value_keys(cls == CLS_U32 ? LC_U32 : cls == CLS_U16 ? LC_U16 : cls == CLS_U8 ? LC_U8 : LC_BIT, q.y,
               cls == CLS_U32 ? 32 * nw : 1, dst);
  } else if (code == CODE_LD_CONST) {
    const uint32_t nw = (q.x >> 12) & 63u;
    value_keys(((q.x >> 18) & 1u) ? LC_BCAST : LC_U32, q.y, 32 * nw, dst);
  } else if (code == CODE_ST_REG || code == CODE_ST_X || code == CODE_ST_OUT || code == CODE_ST_PORT) {
    const uint32_t nw = (q.x >> 12) & 63u, lay = (q.x >> 18) & 7u;
    value_keys(lay, q.y, lay == LC_U32 ? 32 * nw : 32, src);
  } else if (code == CODE_ST_REGC) {
    value_keys((q.x >> 18) & 7u, q.y, q.x >> 21, src);
  }
}
void bit_keys(const BitDesc &q, std::vector<uint64_t> &src, std::vector<uint64_t> &dst) {
  const uint32_t lut = q.x & 0xFFu, immf = q.x >> 8;
  const uint32_t f[3] = {q.y >> 16, q.z & 0xFFFFu, q.z >> 16};
  for (uint32_t k = 0; k < 3; k++)
    if (!(immf & (1u << k)) && lut_uses(lut, k)) src.push_back(skey(SP_S, f[k]));
  dst.push_back(skey(SP_S, q.y & 0xFFFFu));
}

bool jit_compact_env(const Program &G) {
  const char *e = getenv("RTLSIM_JIT_COMPACT");
  return G.L == 1 && (e ? atoi(e) != 0 : true);
}
// forwarding register budget: a slot value is taken from a register only
// within this many descriptors of its write / read. TMEM schedules run 32
// warps at 64 registers and spill; budgets of 4 / 8 / 16
// measured config 4 at 52.8 / 53.0 / 52.9 ms/cycle vs 55.9 unbounded
// (profiles/r02_t_probe_fwd.log, r02_u_probe.log)
uint64_t jit_fwd_ops(bool compact, bool tmem = false) {
  const char *e = getenv("RTLSIM_JIT_FWDOPS");
  if (e) return (uint64_t)atoll(e);
  return compact ? 64u : tmem ? kTmemFwdOps : UINT64_MAX;
}

// (r2) RTLSIM_JIT_UBASE=1: inline step bodies address the state arenas from
// the kernel parameters (uniform, constant bank) plus one 64-bit per-class
// thread offset %to<k>, instead of 16 per-arena 64-bit base registers — the
// registers the 64-per-thread budget of 32-warp TMEM CTAs spills
static_assert(offsetof(JitParams, cur) == 0 && offsetof(JitParams, nxt) == 32 && offsetof(JitParams, xnet) == 64 &&
                  offsetof(JitParams, in) == 96, "jit_ubase reads the arena bases at prm + 32 * arena + 8 * class");
bool jit_ubase() {
  const char *e = getenv("RTLSIM_JIT_UBASE");
  return e && atoi(e) != 0;
}
std::string step_function(const Program &G, const std::string &name, uint32_t s0, uint32_t s1, bool dig,
                          uint32_t nspec, bool to_end, uint32_t *tile_words = nullptr,
                          std::vector<WideRec> *wrec_out = nullptr, std::vector<uint32_t> *bittab_out = nullptr,
                          bool inline_body = false) {
  t_prog = &G;
  const bool compact = jit_compact_env(G) && to_end && tile_words;
  std::vector<Em::Inst> insts;
  std::vector<WideRec> wrec_probe, wrec_final;
  std::vector<uint32_t> bit_probe;
  // dry pass: which warp writes which slot in which step (forwarding validity)
  WriteLog log;
  {
    Em d;
    d.dig = dig;
    d.dry = true;
    d.log = &log;
    for (uint32_t w = 0; w < G.L; w++)
      for (uint32_t s = s0; s < s1; s++) {
        d.warp = w;
        d.step = (int32_t)s;
        std::vector<std::vector<uint32_t>> wb;
        warp_bits(G, s, w, wb);
        for (auto &ch : wb) {
          if (ch.size() >= std::max<uint32_t>(jit_bitany(), 2u)) emit_bit_batch_any(d, G, ch);
          else for (uint32_t k : ch) emit_bit(d, G.bitdesc[k]);
        }
        for (uint32_t k = G.step_ptr[s * G.L + w]; k < G.step_ptr[s * G.L + w + 1]; k++) emit_desc(d, G, G.desc[k]);
      }
  }
  // split-phase barrier: which ops of each (warp, step) may run before the
  // wait for the previous step's barrier (see jit_split)
  const bool split = jit_split() != 0 && G.L > 1;
  std::vector<std::vector<char>> early_bit, early_desc;   // [w * nsteps + (s - s0)][k]
  if (split) {
    const uint32_t ns = s1 - s0;
    early_bit.assign((size_t)G.L * ns, {});
    early_desc.assign((size_t)G.L * ns, {});
    std::unordered_map<uint64_t, std::vector<std::pair<int32_t, uint32_t>>> uses;
    std::vector<uint64_t> src, dst;
    bool ld;
    for (uint32_t w = 0; w < G.L; w++)
      for (uint32_t st = s0; st < s1; st++) {
        for (uint32_t k = G.bit_ptr[st] + w; k < G.bit_ptr[st + 1]; k += G.L) {
          src.clear(); dst.clear();
          bit_keys(G.bitdesc[k], src, dst);
          for (uint64_t x : src) uses[x].push_back({(int32_t)st, w});
        }
        for (uint32_t k = G.step_ptr[st * G.L + w]; k < G.step_ptr[st * G.L + w + 1]; k++) {
          src.clear(); dst.clear();
          desc_keys(G, G.desc[k], src, dst, &ld);
          for (uint64_t x : src) uses[x].push_back({(int32_t)st, w});
        }
      }
    auto is_opaque = [&](uint64_t k, int32_t t, uint32_t w) {
      auto it = log.wo.find(k);
      if (it == log.wo.end()) return false;
      for (auto &x : it->second)
        if (x.first == t && x.second == w) return true;
      return false;
    };
    auto ok = [&](int32_t t, uint32_t w) {
      if (t == (int32_t)s0 || jit_split() == 2) return false;   // 2: A/B, no early ops
      for (uint64_t k : src) {   // the value read: the latest write before step t
        int32_t tw = -1;
        uint32_t ww = 0;
        auto it = log.w.find(k);
        if (it == log.w.end()) return false;
        for (auto &x : it->second)
          if (x.first < t && x.first > tw) tw = x.first, ww = x.second;
        if (tw < 0) return false;
        if (ww == w) continue;                       // this warp's own write
        if (tw > t - 2 || is_opaque(k, tw, ww)) return false;
      }
      for (uint64_t k : dst) {   // no other warp touches the slot in step t - 1
        auto u = uses.find(k);
        if (u != uses.end())
          for (auto &x : u->second)
            if (x.first == t - 1 && x.second != w) return false;
        auto it = log.w.find(k);
        if (it != log.w.end())
          for (auto &x : it->second)
            if (x.first == t - 1 && x.second != w) return false;
      }
      return true;
    };
    static const bool dbg = getenv("RTLSIM_JIT_SPLIT_DEBUG") != nullptr;
    uint64_t n_src_recent = 0, n_src_opq = 0, n_dst = 0, n_ld = 0, n_ok = 0, n_all = 0;
    auto why = [&](int32_t t, uint32_t w) {
      for (uint64_t k : src) {
        int32_t tw = -1; uint32_t ww = 0;
        auto it = log.w.find(k);
        if (it == log.w.end()) continue;
        for (auto &x : it->second) if (x.first < t && x.first > tw) tw = x.first, ww = x.second;
        if (tw >= 0 && ww != w) { if (tw > t - 2) { n_src_recent++; return; } if (is_opaque(k, tw, ww)) { n_src_opq++; return; } }
      }
      n_dst++;
    };
    for (uint32_t w = 0; w < G.L; w++)
      for (uint32_t st = s0; st < s1; st++) {
        auto &eb = early_bit[(size_t)w * ns + (st - s0)];
        auto &ed = early_desc[(size_t)w * ns + (st - s0)];
        for (uint32_t k = G.bit_ptr[st] + w; k < G.bit_ptr[st + 1]; k += G.L) {
          src.clear(); dst.clear();
          bit_keys(G.bitdesc[k], src, dst);
          eb.push_back(ok((int32_t)st, w));
        }
        for (uint32_t k = G.step_ptr[st * G.L + w]; k < G.step_ptr[st * G.L + w + 1]; k++) {
          src.clear(); dst.clear();
          desc_keys(G, G.desc[k], src, dst, &ld);
          ed.push_back(!ld && ok((int32_t)st, w));
          if (dbg && st > s0) {
            n_all++;
            if (ld) n_ld++;
            else if (ed.back()) n_ok++;
            else why((int32_t)st, w);
          }
        }
      }
    if (dbg)
      fprintf(stderr, "split %s: %llu descs, early %llu, loads %llu, late by recent src %llu, opaque src %llu, dst %llu\n",
              name.c_str(), (unsigned long long)n_all, (unsigned long long)n_ok, (unsigned long long)n_ld,
              (unsigned long long)n_src_recent, (unsigned long long)n_src_opq, (unsigned long long)n_dst);
  }
  auto emit_real = [&](Em &e, bool probe, bool dse) {
  e.dig = dig;
  e.dry = false;
  e.probe = probe;
  e.dse = dse;
  e.to_end = to_end;
  e.nspec = nspec;
  e.log = &log;
  e.fwd_max = compact ? INT32_MAX / 2 : jit_fwd_steps();
  e.fwd_ops = jit_fwd_ops(compact, G.tmem_cols != 0);
  e.ubase = inline_body && jit_ubase() && nspec != 0 && G.part_steps.size() > 2;
  e.compact = compact;
  e.inst = &insts;
  e.wrec = probe ? &wrec_probe : &wrec_final;
  e.bittab = probe ? &bit_probe : bittab_out;
  std::vector<std::string> labs(G.L);
  std::string tbl = e.L("T"), end = e.L("E");
  if (G.L > 1) {
    std::string targets;
    for (uint32_t w = 0; w < G.L; w++) {
      labs[w] = e.L("W");
      targets += (w ? ", " : "") + labs[w];
    }
    e.s += tbl + ": .branchtargets " + targets + ";\n";
    e.l(fmt("brx.idx %%wl, %s", tbl.c_str()));
  }
  for (uint32_t w = 0; w < G.L; w++) {
    if (G.L > 1) e.lab(labs[w]);
    e.fwd.clear();
    e.warp = w;
    for (uint32_t s = s0; s < s1; s++) {
      e.step = (int32_t)s;
      if (split) {
        // early ops, the wait for the previous step's barrier, late ops
        const auto &eb = early_bit[(size_t)w * (s1 - s0) + (s - s0)];
        const auto &ed = early_desc[(size_t)w * (s1 - s0) + (s - s0)];
        for (int pass = 0; pass < 2; pass++) {
          if (pass == 1 && s > s0 && jit_split() != 3) {   // 3: code-size probe only (no wait: racy)
            // the wait loop lives in a called function: a loop inside the
            // straight-line code makes ptxas duplicate blocks and add
            // divergence fallbacks around every vote (SASS x1.5 - x2)
            const std::string ra = e.R();
            e.l(fmt("add.u32 %s, %%mbar, %u", ra.c_str(), 8u * ((s - 1) & 1u)));
            e.s += "\t{\n\t.param .b32 mw0;\n\t.param .b64 mw1;\n";
            e.l(fmt("st.param.b32 [mw0], %s", ra.c_str()));
            e.l(fmt("st.param.b64 [mw1], %%mtok%u", (s - 1) & 1u));
            e.l("call.uni rtl_mbar_wait, (mw0, mw1)");
            e.s += "\t}\n";
          }
          uint32_t j = 0;
          for (uint32_t k = G.bit_ptr[s] + w; k < G.bit_ptr[s + 1]; k += G.L, j++) {
            if ((eb[j] != 0) != (pass == 0)) continue;
            const size_t from = e.s.size();
            e.opn++;
            emit_bit(e, G.bitdesc[k]);
            note_kind(e, pass == 0 ? "bit:early" : "bit", from);
          }
          j = 0;
          for (uint32_t k = G.step_ptr[s * G.L + w]; k < G.step_ptr[s * G.L + w + 1]; k++, j++) {
            if ((ed[j] != 0) != (pass == 0)) continue;
            emit_desc(e, G, G.desc[k]);
          }
        }
        e.l("cp.async.commit_group");
        e.l(fmt("cp.async.wait_group %u", G.step_wait[s]));
        if (s + 1 < s1) e.l(fmt("mbarrier.arrive.shared::cta.b64 %%mtok%u, [%%mbar+%u]", s & 1u, 8u * (s & 1u)));
        continue;
      }
      {
        // this warp's bit ops of the step: groups sharing a truth table
        // (immediates folded in) of >= RTLSIM_JIT_BITBATCH ops run
        // lane-parallel, the rest one by one
        const uint32_t bb = jit_bitbatch();
        std::map<uint32_t, std::vector<BitDesc>> groups;
        std::vector<BitDesc> single;
        for (uint32_t k = G.bit_ptr[s] + w; k < G.bit_ptr[s + 1]; k += G.L) {
          if (bb) groups[bit_fold_lut(G.bitdesc[k])].push_back(G.bitdesc[k]);
          else single.push_back(G.bitdesc[k]);
        }
        if (!bb && jit_bitany()) {   // per-lane truth tables (jit_bitany)
          std::vector<std::vector<uint32_t>> wb;
          warp_bits(G, s, w, wb);
          single.clear();
          for (auto &ch : wb) {
            if (ch.size() >= std::max<uint32_t>(jit_bitany(), 2u)) {
              const size_t from = e.s.size();
              e.opn += ch.size();
              emit_bit_batch_any(e, G, ch);
              note_kind(e, "bitany", from);
            } else {
              for (uint32_t k : ch) single.push_back(G.bitdesc[k]);
            }
          }
        }
        for (auto &g : groups) {
          if (g.second.size() < bb) {
            single.insert(single.end(), g.second.begin(), g.second.end());
            continue;
          }
          for (size_t i = 0; i < g.second.size(); i += 32) {
            std::vector<BitDesc> part(g.second.begin() + i, g.second.begin() + std::min(g.second.size(), i + 32));
            const size_t from = e.s.size();
            e.opn += part.size();
            emit_bit_batch(e, part, g.first);
            note_kind(e, "bitbatch", from);
          }
        }
        for (const BitDesc &q : single) {
          const size_t from = e.s.size();
          e.opn++;
          emit_bit(e, q);
          note_kind(e, "bit", from);
        }
      }
      for (uint32_t k0 = G.step_ptr[s * G.L + w], k = k0; k < G.step_ptr[s * G.L + w + 1]; k++) {
        const uint32_t g = jit_tmgroup();
        if (G.tmem_cols && g > 1 && e.fwd_max > 0 && (k - k0) % g == 0) {
          std::vector<uint32_t> cols;
          for (uint32_t j = k; j < std::min<uint32_t>(k + g, G.step_ptr[s * G.L + w + 1]); j++)
            tm_cols_of(e, G, G.desc[j], cols);
          tm_prefetch_cols(e, cols);
        }
        emit_desc(e, G, G.desc[k]);
      }
      e.l("cp.async.commit_group");
      e.l(fmt("cp.async.wait_group %u", G.step_wait[s]));
      // The per-warp code blocks each hold their own copy of the step
      // barrier, so different warps reach barrier 0 through different
      // barrier instructions. ADVICE r1 asked for the non-.aligned form
      // (barrier.sync) there; measured, it makes ptxas treat every step as
      // potentially divergent: config 3 partition 0 grows from 21,272 to
      // 48,208 SASS instructions (WARPSYNC before every vote and barrier) and
      // runs slower. Every warp of the CTA executes exactly one barrier-0
      // instruction per step, warp-converged, in the same order — the
      // property the hardware barrier counts, and the one warp-specialised
      // CUTLASS kernels rely on when producer and consumer warps meet at a
      // named barrier from different code. The aligned form is kept;
      // RTLSIM_JIT_TBAR=2 emits the non-aligned one for A/B.
      // (r2) TMEM values: this warp's tcgen05.st complete and ordered before
      // the barrier, other warps' after it (fence / sync / fence)
      if (G.tmem_cols) {
        e.l("tcgen05.wait::st.sync.aligned");
        e.l("tcgen05.fence::before_thread_sync");
      }
      if (jit_tbar() == 0)
        e.l("bar.sync 0");
      else if (jit_tbar() == 2)
        e.l("barrier.sync 0");
      else if (G.L > 1)
        e.l(fmt("bar.sync %%tbar, %u", 32u * G.L));   // aligned: one per step in every warp of the tile
      else
        e.l("bar.warp.sync -1");
      if (G.tmem_cols) e.l("tcgen05.fence::after_thread_sync");
    }
    if (G.L > 1) e.l(fmt("bra.uni %s", end.c_str()));
  }
  e.lab(end);
  };
  // dead slot-store elimination (RTLSIM_JIT_DSE, default on; =0 for A/B): a probe pass
  // records which slot reads still go to shared memory once forwarding is
  // applied; the final pass drops the stores nobody reads from there
  Em e;
  if (jit_dse() || compact) {
    Em pe;
    emit_real(pe, true, false);
    if (compact) {
      // first-fit by step interval over the instances read back from shared
      // memory (or written opaquely); space is reused only across steps, so
      // a cp.async into a reused row never overtakes a read of its old value
      std::vector<uint32_t> order;
      for (uint32_t i = 0; i < insts.size(); i++)
        if (insts[i].need) order.push_back(i);
      std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
        return insts[a].s0 != insts[b].s0 ? insts[a].s0 < insts[b].s0 : a < b;
      });
      struct Act { uint32_t nb, words; int32_t s1; };
      std::vector<Act> act;
      uint32_t extent = 0;
      for (uint32_t id : order) {
        Em::Inst &I = insts[id];
        act.erase(std::remove_if(act.begin(), act.end(), [&](const Act &a) { return a.s1 < I.s0; }), act.end());
        std::sort(act.begin(), act.end(), [](const Act &a, const Act &b) { return a.nb < b.nb; });
        uint32_t at = 0;
        for (const Act &a : act) {
          if (a.nb >= at + I.words) break;
          at = std::max(at, a.nb + a.words);
        }
        I.nb = at;
        act.push_back({at, I.words, std::max(I.s0, I.s1)});
        extent = std::max(extent, at + I.words);
      }
      *tile_words = extent;
      if (getenv("RTLSIM_JIT_COMPACT_DEBUG")) {
        std::map<int32_t, std::array<uint64_t, 3>> live;   // step -> words (all, loaded, reread)
        for (uint32_t id : order) {
          const Em::Inst &I = insts[id];
          for (int32_t t = I.s0; t <= std::max(I.s0, I.s1); t++) {
            live[t][0] += I.words;
            if (I.opq) live[t][1] += I.words;
          }
        }
        uint64_t mx = 0, ml = 0;
        for (auto &kv : live)
          if (kv.second[0] > mx) mx = kv.second[0], ml = kv.second[1];
        size_t n_need = order.size();
        fprintf(stderr, "compact %s: %zu instances, %zu in smem, extent %u words, peak live %llu words (%llu loaded)\n",
                name.c_str(), insts.size(), n_need, extent, (unsigned long long)mx, (unsigned long long)ml);
      }
    }
    emit_real(e, false, true);
    if (compact && wrec_out) *wrec_out = wrec_final;
  } else {
    emit_real(e, false, false);
  }
  // (r2) inline_body: the same code as a block of the kernel (no call: no
  // parameter passing, no caller stack frame, one register allocation)
  std::string out = inline_body ? std::string("\t{\n") : func_proto(name) + "\n{\n";
  out += fmt("\t.reg .b32 %%r<%u>;\n\t.reg .b64 %%rd<%u>;\n\t.reg .pred %%p<%u>;\n", e.nr + 1, e.nrd + 1, e.np + 1);
  out += "\t.reg .b64 %mtok0, %mtok1;\n";
  out += "\t.reg .b32 %rq2, %rq3, %rq4;\n";
  if (inline_body) {
    out += "\t.reg .b32 %rw, %rh, %rb, %N4, %N2, %Nb, %lsh;\n\t.reg .b64 %tbb1, %tbb2, %tlw";
  } else {
    out += "\t.reg .b32 %smb, %lane, %wl, %N, %tbar, %mbar, %tmt, %rw, %rh, %rb, %N4, %N2, %Nb, %lsh;\n\t.reg .b64 %tbb1, %tbb2, %tlw, ";
    for (int i = 0; i < kN64; i++) out += fmt("%s%%%s", i ? ", " : "", kCtx64[i]);
  }
  out += ";\n\t.reg .pred %pl0, %pl8, %pl16, %pl24, %pdig;\n\t.reg .b32 %vsm;\n\t.reg .b64 %vdl;\n";
  if (!inline_body) {
    for (int i = 0; i < kN32; i++) out += fmt("\tld.param.u32 %%%s, [a_%s];\n", kCtx32[i], kCtx32[i]);
    for (int i = 0; i < kN64; i++) out += fmt("\tld.param.u64 %%%s, [a_%s];\n", kCtx64[i], kCtx64[i]);
  }
  out += "\tmad.lo.u32 %rq2, %lane, 8, %smb;\n\tmad.lo.u32 %rq3, %lane, 12, %smb;\n\tmad.lo.u32 %rq4, %lane, 16, %smb;\n";
  out += "\tmad.lo.u32 %rw, %lane, 4, %smb;\n\tmad.lo.u32 %rh, %lane, 2, %smb;\n\tadd.u32 %rb, %lane, %smb;\n"
         "\tshl.b32 %N4, %N, 2;\n\tshl.b32 %N2, %N, 1;\n\tshr.u32 %Nb, %N, 3;\n"
         "\tsetp.eq.u32 %pl0, %lane, 0;\n\tsetp.lt.u32 %pl8, %lane, 8;\n\tsetp.lt.u32 %pl16, %lane, 16;\n"
         "\tsetp.ne.u64 %pdig, %dig, 0;\n\tsub.u32 %lsh, 31, %lane;\n"
         "\tmul.wide.u32 %tlw, %lane, 3;\n\tsub.s64 %tbb1, %tb_n1, %tlw;\n"
         "\tmul.wide.u32 %tlw, %lane, 2;\n\tsub.s64 %tbb2, %tb_n2, %tlw;\n";
  if (e.used_v)   // 16-byte wide loads: smem / global offsets of lane l (row l >> 3, bytes 16 (l & 7))
    out += "\tsetp.lt.u32 %pl24, %lane, 24;\n\t{\n\t.reg .b32 %vq, %vr;\n\t.reg .b64 %vw;\n"
           "\tshr.u32 %vq, %lane, 3;\n\tand.b32 %vr, %lane, 7;\n"
           "\tmad.lo.u32 %vsm, %vq, 128, %smb;\n\tmad.lo.u32 %vsm, %vr, 16, %vsm;\n"
           "\tmul.wide.u32 %vdl, %vq, %N4;\n\tmul.wide.u32 %vw, %vr, 16;\n\tadd.s64 %vdl, %vdl, %vw;\n"
           "\tmul.wide.u32 %vw, %lane, 4;\n\tsub.s64 %vdl, %vdl, %vw;\n\t}\n";
  out += e.s;
  out += inline_body ? "\t}\n" : "\tret;\n}\n";
  return out;
}
bool jit_inline() {
  const char *e = getenv("RTLSIM_JIT_INLINE");
  return e ? atoi(e) != 0 : jit_ubase();
}

}  // namespace

bool jit_compact(const Program &G) { return jit_compact_env(G); }

std::string jit_partition_ptx(const Program &G, uint32_t q, const std::string &rt_ptx, uint32_t tmax, bool dig,
                              uint32_t nspec, JitPartInfo *info) {
  const bool compact = jit_compact_env(G);
  const uint32_t s0 = G.part_steps[q], s1 = G.part_steps[q + 1];
  std::string mod;
  mod.reserve(1 << 20);
  mod += ".version 8.8\n.target sm_100a\n.address_size 64\n\n";
  mod += rt_ptx;
  mod += "\n.extern .shared .align 16 .b8 dyn_smem[];\n\n";
  if (jit_vwide()) mod += kVShiftPtx;
  // wait for a phase of a split-phase step barrier (jit_split)
  mod += ".func rtl_mbar_wait(.param .b32 mb_a, .param .b64 mb_t)\n{\n\t.reg .b32 %ra;\n\t.reg .b64 %rt;\n"
         "\t.reg .pred %pw;\n\tld.param.b32 %ra, [mb_a];\n\tld.param.b64 %rt, [mb_t];\n$MBW:\n"
         "\tmbarrier.try_wait.shared::cta.b64 %pw, [%ra], %rt;\n\t@!%pw bra.uni $MBW;\n\tret;\n}\n\n";
  // step groups of bounded size (ptxas time is superlinear in function size).
  // Default: one function per partition. With several called functions
  // ptxas keeps the global-memory descriptor in a uniform register only in
  // the first one; the others hold it in a GPR pair and issue two R2UR
  // before every LDGSTS/STG (~10 % of their SASS, config 3). 1600 ops per
  // function was 2-5 % faster than 800, 800 5-10 % faster than 400.
  std::vector<std::pair<uint32_t, uint32_t>> groups;
  static const uint64_t kGroupOps =
      getenv("RTLSIM_JIT_GROUP") ? strtoull(getenv("RTLSIM_JIT_GROUP"), nullptr, 10) : (1ull << 40);
  uint32_t g0 = s0;
  uint64_t acc = 0;
  for (uint32_t s = s0; s < s1; s++) {
    acc += (G.step_ptr[(s + 1) * G.L] - G.step_ptr[s * G.L]) + (G.bit_ptr[s + 1] - G.bit_ptr[s]);
    // compacted slots are allocated per function: one function per partition
    if ((acc >= kGroupOps && !compact) || s + 1 == s1) {
      groups.push_back({g0, s + 1});
      g0 = s + 1;
      acc = 0;
    }
  }
  uint32_t tile_words = 0;
  JitPartInfo local;
  if (!info) info = &local;
  const bool inl = jit_inline();
  std::vector<std::string> bodies;
  for (size_t g = 0; g < groups.size(); g++) {
    std::string f = step_function(G, fmt("rtl_steps_%zu", g), groups[g].first, groups[g].second, dig, nspec,
                                  groups[g].second == s1, compact ? &tile_words : nullptr,
                                  compact ? &info->wide : nullptr, &info->bittab, inl);
    if (inl) bodies.push_back(std::move(f));
    else mod += f + "\n";
  }
  // shared memory per tile: the compacted extent, or the schedule's slots
  const uint32_t tbytes = compact ? std::max<uint32_t>(16u, ((tile_words * 4u) + 15u) & ~15u) : jit_tile_bytes(G);
  info->tile_bytes = tbytes;
  // the kernel: per-thread context, then the step functions in order
  // A CTA holds `tpc` tiles; warp g works on tile g / L as op-lane g % L, so
  // the warps of one op-lane (one per tile) run identical code in step
  // lock-step and share its instruction fetch.
  mod += fmt(".visible .entry rtl_jit_part(.param .align 8 .b8 prm[%zu])\n.maxntid %u, 1, 1\n{\n",
             sizeof(JitParams), 32u * G.L * (G.tmem_cols ? 4u : std::max<uint32_t>(tmax, 1u)));
  mod += "\t.reg .b32 %tidx, %tile, %s, %smb, %lane, %wl, %N, %wg, %tsub, %tpc, %tbar, %mbar, %nthr, %tmt, %tmb;\n\t.reg .b64 %t64, %b64, %digb;\n\t.reg .pred %pz, %pw0;\n\t.reg .b64 ";
  for (int i = 0; i < kN64; i++) mod += fmt("%s%%%s", i ? ", " : "", kCtx64[i]);
  mod += ";\n";
  if (G.tmem_cols)
    // (r2) TMEM mode: 4 tiles per CTA, tile t on lane quarter / SMSP t (warp
    // w: tile w & 3, op-lane w >> 2) — a warp reaches only its quarter's lanes
    mod += "\tmov.u32 %tidx, %tid.x;\n\tand.b32 %lane, %tidx, 31;\n\tshr.u32 %wg, %tidx, 5;\n"
           "\tshr.u32 %wl, %wg, 2;\n\tand.b32 %tsub, %wg, 3;\n";
  else
    mod += fmt("\tmov.u32 %%tidx, %%tid.x;\n\tand.b32 %%lane, %%tidx, 31;\n\tshr.u32 %%wg, %%tidx, 5;\n"
               "\trem.u32 %%wl, %%wg, %u;\n\tdiv.u32 %%tsub, %%wg, %u;\n", G.L, G.L);
  mod += "\tsetp.lt.u32 %pw0, %tidx, 32;\n\tmov.u32 %tmt, 0;\n\tmov.u32 %tmb, 0;\n";
  mod += fmt("\tld.param.u32 %%tpc, [prm+%zu];\n", offsetof(JitParams, tpc));
  mod += "\tadd.u32 %tbar, %tsub, 1;\n";
  mod += "\tmov.u32 %tile, %ctaid.x;\n\tmad.lo.u32 %tile, %tile, %tpc, %tsub;\n\tmad.lo.u32 %s, %tile, 32, %lane;\n";
  mod += fmt("\tld.param.u32 %%N, [prm+%zu];\n", offsetof(JitParams, N));
  if (nspec)   // row offsets are immediates for this N_pad: refuse any other
    mod += fmt("\t{\n\t.reg .pred %%pn;\n\tsetp.ne.u32 %%pn, %%N, %u;\n\t@%%pn trap;\n\t}\n", nspec);
  // per-class 64-bit thread offsets into an arena (tile * row bytes + lane
  // * 4; bit rows: tile * 4) for the parameter-based addressing (jit_ubase)
  mod += "\t.reg .b64 %to0, %to1, %to2, %to3;\n";
  {
    const uint32_t tm[4] = {4, 32, 64, 128};
    for (int k = 0; k < 4; k++) {
      mod += fmt("\tmul.wide.u32 %%to%d, %%tile, %u;\n", k, tm[k]);
      if (k > 0) mod += fmt("\tmul.wide.u32 %%t64, %%lane, 4;\n\tadd.u64 %%to%d, %%to%d, %%t64;\n", k, k);
    }
  }
  const size_t aoff[4] = {offsetof(JitParams, cur), offsetof(JitParams, nxt), offsetof(JitParams, xnet),
                          offsetof(JitParams, in)};
  const char *tag[4] = {"c", "n", "x", "i"};
  for (int A = 0; A < 4; A++) {
    // bit rows: + tile*4 ; u8: + tile*32 + lane*4 ; u16: + tile*64 + lane*4 ; u32: + tile*128 + lane*4
    const uint32_t tmul[4] = {4, 32, 64, 128};
    for (int k = 0; k < 4; k++) {
      mod += fmt("\tld.param.u64 %%b64, [prm+%zu];\n", aoff[A] + 8 * k);
      mod += fmt("\tmul.wide.u32 %%t64, %%tile, %u;\n\tadd.u64 %%tb_%s%d, %%b64, %%t64;\n", tmul[k], tag[A], k);
      if (k > 0) mod += fmt("\tmul.wide.u32 %%t64, %%lane, 4;\n\tadd.u64 %%tb_%s%d, %%tb_%s%d, %%t64;\n", tag[A], k, tag[A], k);
    }
  }
  mod += fmt("\tld.param.u64 %%b64, [prm+%zu];\n\tmul.wide.u32 %%t64, %%s, 4;\n\tadd.u64 %%outb, %%b64, %%t64;\n",
             offsetof(JitParams, out));
  mod += fmt("\tld.param.u64 %%digb, [prm+%zu];\n\tmul.wide.u32 %%t64, %%s, 8;\n\tadd.u64 %%t64, %%digb, %%t64;\n"
             "\tsetp.eq.u64 %%pz, %%digb, 0;\n\tselp.b64 %%dig, 0, %%t64, %%pz;\n",
             offsetof(JitParams, digest));
  mod += fmt("\tld.param.u64 %%wide, [prm+%zu];\n", offsetof(JitParams, wide));
  mod += fmt("\tld.param.u64 %%b64, [prm+%zu];\n\tmul.wide.u32 %%t64, %%lane, 16;\n\tadd.u64 %%bitl, %%b64, %%t64;\n",
             offsetof(JitParams, bittab));
  // memory / write-port arenas: this stimulus' column ([row][N_pad] u32)
  mod += fmt("\tld.param.u64 %%b64, [prm+%zu];\n\tmul.wide.u32 %%t64, %%s, 4;\n\tadd.u64 %%memb, %%b64, %%t64;\n",
             offsetof(JitParams, mem));
  mod += fmt("\tld.param.u64 %%b64, [prm+%zu];\n\tadd.u64 %%portb, %%b64, %%t64;\n", offsetof(JitParams, port));
  // the split-phase step barrier pair after the CTA's tiles (16 bytes)
  mod += fmt("\tmov.u32 %%mbar, dyn_smem;\n\tmad.lo.u32 %%mbar, %%tpc, %u, %%mbar;\n", tbytes);
  if (jit_split() != 0 && G.L > 1)
    mod += "\tmov.u32 %nthr, %ntid.x;\n\t{\n\t.reg .pred %p0;\n\tsetp.eq.u32 %p0, %tidx, 0;\n"
           "\t@%p0 mbarrier.init.shared::cta.b64 [%mbar], %nthr;\n\t@%p0 mbarrier.init.shared::cta.b64 [%mbar+8], %nthr;\n"
           "\tbar.sync 0;\n\t}\n";
  mod += fmt("\tmov.u32 %%smb, dyn_smem;\n\tmad.lo.u32 %%smb, %%tsub, %u, %%smb;\n\tcvta.shared.u64 %%smg, dyn_smem;\n"
             "\tmul.wide.u32 %%t64, %%tsub, %u;\n\tadd.u64 %%smg, %%smg, %%t64;\n",
             tbytes, tbytes);
  uint32_t tcols = 32;   // TMEM allocation: a power of two >= 32 columns
  while (tcols < G.tmem_cols) tcols *= 2;
  if (G.tmem_cols) {
    // (r2) warp 0 allocates the TMEM columns (one CTA per SM: the tiles
    // fill the shared memory) and publishes the base after the split-barrier
    // pair; lane quarter t of the allocation belongs to tile t
    mod += "\t{\n\t.reg .b32 %ta;\n\tadd.u32 %ta, %mbar, 16;\n";
    mod += fmt("\t@%%pw0 tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%%ta], %u;\n", tcols);
    mod += "\t@%pw0 tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n"
           "\ttcgen05.fence::before_thread_sync;\n\tbar.sync 0;\n\ttcgen05.fence::after_thread_sync;\n"
           "\tld.shared.u32 %tmb, [%ta];\n\tshl.b32 %ta, %tsub, 21;\n\tadd.u32 %tmt, %tmb, %ta;\n\t}\n";
  }
  // M1 cycle loop (nc > 1, single-partition designs only): after each cycle
  // the state buffers swap, the input / output / digest rows advance, and a
  // CTA barrier orders this cycle's register stores before the next cycle's
  // loads (the tile's stimuli are its own: no other CTA is involved)
  mod += "\t{\n\t.reg .b32 %cyc, %ncy;\n\t.reg .b64 %tsw, %stp;\n\t.reg .pred %pcy;\n";
  mod += fmt("\tld.param.u32 %%ncy, [prm+%zu];\n\tmov.u32 %%cyc, 0;\n$CYC:\n", offsetof(JitParams, nc));
  for (size_t g = 0; g < groups.size(); g++) {
    if (inl) {
      mod += bodies[g];
      continue;
    }
    mod += "\t{\n";
    std::string args;
    int pi = 0;
    for (int i = 0; i < kN32; i++, pi++) {
      mod += fmt("\t.param .b32 q%d;\n\tst.param.b32 [q%d], %%%s;\n", pi, pi, kCtx32[i]);
      args += fmt("%sq%d", pi ? ", " : "", pi);
    }
    for (int i = 0; i < kN64; i++, pi++) {
      mod += fmt("\t.param .b64 q%d;\n\tst.param.b64 [q%d], %%%s;\n", pi, pi, kCtx64[i]);
      args += fmt(", q%d", pi);
    }
    mod += fmt("\tcall.uni rtl_steps_%zu, (%s);\n\t}\n", g, args.c_str());
  }
  mod += "\tadd.u32 %cyc, %cyc, 1;\n\tsetp.lt.u32 %pcy, %cyc, %ncy;\n\t@!%pcy bra.uni $CYCE;\n";
  for (int k = 0; k < 4; k++) {
    mod += fmt("\tmov.u64 %%tsw, %%tb_c%d;\n\tmov.u64 %%tb_c%d, %%tb_n%d;\n\tmov.u64 %%tb_n%d, %%tsw;\n", k, k, k, k);
    mod += fmt("\tld.param.u64 %%stp, [prm+%zu];\n\tadd.u64 %%tb_i%d, %%tb_i%d, %%stp;\n",
               offsetof(JitParams, in_step) + 8 * k, k, k);
  }
  mod += fmt("\tld.param.u64 %%stp, [prm+%zu];\n\tadd.u64 %%outb, %%outb, %%stp;\n", offsetof(JitParams, out_step));
  mod += fmt("\tld.param.u64 %%stp, [prm+%zu];\n\tsetp.ne.u64 %%pcy, %%dig, 0;\n\t@%%pcy add.u64 %%dig, %%dig, %%stp;\n",
             offsetof(JitParams, dig_step));
  mod += "\tbar.sync 0;\n\tbra.uni $CYC;\n$CYCE:\n\t}\n";
  if (G.tmem_cols)
    mod += "\ttcgen05.fence::before_thread_sync;\n\tbar.sync 0;\n\ttcgen05.fence::after_thread_sync;\n" +
           fmt("\t@%%pw0 tcgen05.dealloc.cta_group::1.sync.aligned.b32 %%tmb, %u;\n", tcols);
  mod += "\tret;\n}\n";
  return mod;
}

// SASS instructions in a cubin: the sizes of its .text.* sections (ELF64) /
// 16 bytes per Blackwell instruction
static uint64_t cubin_sass_instructions(const std::vector<char> &b) {
  if (b.size() < 64 || memcmp(b.data(), "\x7f" "ELF", 4) != 0 || b[4] != 2) return 0;
  auto u16 = [&](size_t o) { uint16_t v; memcpy(&v, b.data() + o, 2); return v; };
  auto u32 = [&](size_t o) { uint32_t v; memcpy(&v, b.data() + o, 4); return v; };
  auto u64 = [&](size_t o) { uint64_t v; memcpy(&v, b.data() + o, 8); return v; };
  const uint64_t shoff = u64(0x28);
  const uint16_t shentsize = u16(0x3A), shnum = u16(0x3C), shstrndx = u16(0x3E);
  if (shoff + (uint64_t)shnum * shentsize > b.size() || shstrndx >= shnum) return 0;
  const uint64_t stroff = u64(shoff + (uint64_t)shstrndx * shentsize + 0x18);
  uint64_t total = 0;
  for (uint16_t i = 0; i < shnum; i++) {
    const size_t h = shoff + (size_t)i * shentsize;
    const uint64_t name = stroff + u32(h);
    if (name + 6 > b.size()) continue;
    if (strncmp(b.data() + name, ".text.", 6) == 0) total += u64(h + 0x20);
  }
  return total / 16;
}

static int compile_ptx(const std::string &ptx, bool o3, std::vector<char> *cubin, std::string *err) {
  nvPTXCompilerHandle h = nullptr;
  if (nvPTXCompilerCreate(&h, ptx.size(), ptx.c_str()) != NVPTXCOMPILE_SUCCESS) {
    *err = "nvPTXCompilerCreate failed";
    return -1;
  }
  // --Ofast-compile=mid: ~3x faster than -O3 on this straight-line code for
  // ~2% more SASS (measured on the riscv-mini-shaped design)
  const char *opts[] = {"--gpu-name=sm_100a", o3 ? "-O3" : "--Ofast-compile=mid"};
  nvPTXCompileResult rc = nvPTXCompilerCompile(h, 2, opts);
  if (rc != NVPTXCOMPILE_SUCCESS) {
    size_t n = 0;
    nvPTXCompilerGetErrorLogSize(h, &n);
    std::string log(n, '\0');
    if (n) nvPTXCompilerGetErrorLog(h, &log[0]);
    *err = "ptx compile failed: " + log.substr(0, 2000);
    nvPTXCompilerDestroy(&h);
    return -1;
  }
  size_t n = 0;
  nvPTXCompilerGetCompiledProgramSize(h, &n);
  cubin->resize(n);
  nvPTXCompilerGetCompiledProgram(h, cubin->data());
  nvPTXCompilerDestroy(&h);
  return 0;
}

int jit_build(const Program &G, const std::string &rt_ptx_path, uint32_t smem_bytes, int device, JitKernels *out,
              std::string *err, bool dig, uint32_t nspec) {
  std::ifstream f(rt_ptx_path);
  if (!f) {
    *err = "cannot read " + rt_ptx_path;
    return RTLSIM_E_ARG;
  }
  std::stringstream ss;
  ss << f.rdbuf();
  // strip the header lines (.version/.target/.address_size) of the runtime PTX
  std::string rt, line;
  std::istringstream is(ss.str());
  while (std::getline(is, line)) {
    if (line.rfind(".version", 0) == 0 || line.rfind(".target", 0) == 0 || line.rfind(".address_size", 0) == 0) continue;
    rt += line + "\n";
  }
  const uint32_t NP = (uint32_t)G.part_steps.size() - 1;
  // tiles per CTA the kernels are built for (their thread count bounds registers)
  // (compacted kernels: their shared memory is known only after generation;
  // the launch picks the tiles per CTA that fit, up to tmax)
  const bool compact = jit_compact_env(G);
  const uint32_t tmax = compact
      ? std::max<uint32_t>(1u, std::min<uint32_t>(jit_default_tiles(true), 32u))
      : std::max<uint32_t>(
            1u, std::min<uint32_t>(std::min<uint32_t>(jit_default_tiles(), 32u / std::max<uint32_t>(G.L, 1u)),
                                   smem_bytes / jit_tile_bytes(G)));
  out->tmax = G.tmem_cols ? 4u : tmax;   // TMEM: four tiles, one per lane quarter
  out->compact = compact;
  std::vector<JitPartInfo> infos(NP);
  out->nspec = nspec;
  // ptxas -O3 schedules this code better than --Ofast-compile=mid (config 3
  // ~1.8x, config 4 175 vs 185 ms/cycle) but compiles ~3x slower (config 4:
  // 116 s on 16 cores); the cubin cache amortises it (RTLSIM_JIT_OPT=O3 / mid
  // overrides)
  const uint64_t nops = G.desc.size() + G.bitdesc.size();
  const char *lvl = getenv("RTLSIM_JIT_OPT");
  const bool o3 = lvl ? strcmp(lvl, "O3") == 0 : nops <= 2000000;
  out->o3 = o3;
  out->kern.assign(NP, nullptr);
  out->libs.assign(NP, nullptr);
  std::vector<std::vector<char>> cubins(NP);
  std::vector<std::string> errs(NP);
  std::vector<char> from_cache(NP, 0);
  std::atomic<uint32_t> next{0};
  std::atomic<size_t> ptx_bytes{0};
  std::atomic<uint32_t> cache_hits{0};
  // RTLSIM_JIT_CACHE=dir: a private cubin cache. It is used only when it is
  // a directory owned by this user and not writable by anyone else (cubins
  // found there are loaded and run in this process); otherwise the
  // kernels are compiled without a cache.
  std::string cache_dir;
  if (const char *cdir = getenv("RTLSIM_JIT_CACHE"))
    if (*cdir) {
      mkdir(cdir, 0700);   // one level; an existing directory is checked below
      struct stat sb;
      if (stat(cdir, &sb) == 0 && S_ISDIR(sb.st_mode) && sb.st_uid == geteuid() && !(sb.st_mode & 022))
        cache_dir = cdir;
    }
  auto t0 = std::chrono::steady_clock::now();
  unsigned nth = std::max(1u, std::thread::hardware_concurrency());
  std::vector<std::thread> th;
  for (unsigned t = 0; t < std::min<unsigned>(nth, NP ? NP : 1); t++) {
    th.emplace_back([&]() {
      for (uint32_t q; (q = next++) < NP;) {
        if (G.part_steps[q] == G.part_steps[q + 1]) continue;
        // debugging aid (host-only inspection): RTLSIM_JIT_ONLY=q emits one partition
        if (getenv("RTLSIM_JIT_ONLY") && (uint32_t)atoi(getenv("RTLSIM_JIT_ONLY")) != q) continue;
        std::string ptx = jit_partition_ptx(G, q, rt, tmax, dig, nspec, &infos[q]);
        ptx_bytes += ptx.size();
        if (const char *dir = getenv("RTLSIM_JIT_SAVE")) {   // debugging aid: keep the module
          std::ofstream o(fmt("%s/part%u.ptx", dir, q));
          o << ptx;
        }
        // RTLSIM_JIT_CACHE=dir: cubins keyed by a hash of (PTX, options);
        // lets the ranks of one node (bench.py) and repeated loads share work
        const char *cdir = cache_dir.c_str();
        std::string cpath;
        if (!cache_dir.empty()) {
          uint64_t h = 1469598103934665603ull;   // FNV-1a
          auto mixin = [&](const std::string &x) {
            for (unsigned char ch : x) h = (h ^ ch) * 1099511628211ull;
          };
          mixin(ptx);
          mixin(o3 ? "|O3|sm_100a" : "|mid|sm_100a");
          cpath = fmt("%s/%016llx.cubin", cdir, (unsigned long long)h);
          std::ifstream in(cpath, std::ios::binary);
          if (in) {
            std::vector<char> buf((std::istreambuf_iterator<char>(in)), std::istreambuf_iterator<char>());
            if (!buf.empty()) {
              cubins[q] = std::move(buf);
              from_cache[q] = 1;
              cache_hits++;
              continue;
            }
          }
        }
        if (compile_ptx(ptx, o3, &cubins[q], &errs[q]) != 0) {
          if (getenv("RTLSIM_JIT_DUMP")) {
            std::ofstream o(fmt("/tmp/rtlsim_jit_fail_%u.ptx", q));
            o << ptx;
          }
        } else if (!cpath.empty()) {
          const std::string tmp = cpath + fmt(".tmp%d.%u", (int)getpid(), q);
          bool ok;
          {
            std::ofstream o(tmp, std::ios::binary);
            o.write(cubins[q].data(), (std::streamsize)cubins[q].size());
            o.flush();
            ok = (bool)o;
          }
          // only a complete file is published under the cache name
          if (ok) ok = std::rename(tmp.c_str(), cpath.c_str()) == 0;
          if (!ok) std::remove(tmp.c_str());
        }
      }
    });
  }
  for (auto &t : th) t.join();
  auto t1 = std::chrono::steady_clock::now();
  out->compile_s = std::chrono::duration<double>(t1 - t0).count();
  out->ptx_bytes = ptx_bytes;
  out->cache_hits = cache_hits;
  for (uint32_t q = 0; q < NP; q++)
    if (!errs[q].empty()) {
      *err = fmt("partition %u: ", q) + errs[q];
      return RTLSIM_E_ARG;
    }
  out->tile_bytes.assign(NP, 0);
  out->wide_base.assign(NP, 0);
  std::vector<WideRec> wall;
  for (uint32_t q = 0; q < NP; q++) {
    out->tile_bytes[q] = infos[q].tile_bytes ? infos[q].tile_bytes : jit_tile_bytes(G);
    out->wide_base[q] = (uint32_t)wall.size();
    wall.insert(wall.end(), infos[q].wide.begin(), infos[q].wide.end());
  }
  std::vector<uint32_t> ball;
  out->bit_base.assign(NP, 0);
  for (uint32_t q = 0; q < NP; q++) {
    out->bit_base[q] = (uint32_t)(ball.size() / 4);
    ball.insert(ball.end(), infos[q].bittab.begin(), infos[q].bittab.end());
  }
  if (device >= 0 && !ball.empty()) {
    cudaError_t e = cudaMalloc((void **)&out->d_bittab, ball.size() * 4);
    if (e == cudaSuccess) e = cudaMemcpy(out->d_bittab, ball.data(), ball.size() * 4, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      *err = std::string("JIT bit-op table: ") + cudaGetErrorString(e);
      cudaGetLastError();
      return RTLSIM_E_CUDA;
    }
  }
  if (device >= 0 && !wall.empty()) {
    cudaError_t e = cudaMalloc((void **)&out->d_wide, wall.size() * sizeof(WideRec));
    if (e == cudaSuccess) e = cudaMemcpy(out->d_wide, wall.data(), wall.size() * sizeof(WideRec), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      *err = std::string("JIT record table: ") + cudaGetErrorString(e);
      cudaGetLastError();
      return RTLSIM_E_CUDA;
    }
  }
  for (uint32_t q = 0; q < NP; q++) {
    if (cubins[q].empty()) continue;
    out->cubin_bytes += cubins[q].size();
    out->sass_instructions += cubin_sass_instructions(cubins[q]);
    if (device < 0) continue;
    cudaError_t e = cudaLibraryLoadData(&out->libs[q], cubins[q].data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
    if (e != cudaSuccess && from_cache[q]) {   // a damaged cached cubin: compile it again
      cudaGetLastError();
      std::string cerr;
      if (compile_ptx(jit_partition_ptx(G, q, rt, tmax, dig, nspec, &infos[q]), o3, &cubins[q], &cerr) != 0) {
        *err = fmt("partition %u: ", q) + cerr;
        return RTLSIM_E_ARG;
      }
      e = cudaLibraryLoadData(&out->libs[q], cubins[q].data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
    }
    if (e == cudaSuccess) e = cudaLibraryGetKernel(&out->kern[q], out->libs[q], "rtl_jit_part");
    if (e == cudaSuccess) {   // the launch picks tiles per CTA within the device's opt-in maximum
      int optin = (int)std::max<uint32_t>(smem_bytes, 1024);
      cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
      e = cudaKernelSetAttributeForDevice(out->kern[q], cudaFuncAttributeMaxDynamicSharedMemorySize, optin, device);
    }
    if (e != cudaSuccess) {
      *err = std::string("loading JIT kernel: ") + cudaGetErrorString(e);
      cudaGetLastError();
      return RTLSIM_E_CUDA;
    }
  }
  return RTLSIM_OK;
}

uint32_t jit_default_tiles(bool compact) {
  const char *e = getenv("RTLSIM_JIT_TMAX");   // read per load (tests vary it)
  return e ? std::min<uint32_t>(kJitMaxTiles, (uint32_t)std::max(1, atoi(e))) : (compact ? 16u : 4u);
}

void jit_free(JitKernels *k) {
  if (k->d_wide) cudaFree(k->d_wide);
  k->d_wide = nullptr;
  if (k->d_bittab) cudaFree(k->d_bittab);
  k->d_bittab = nullptr;
  for (cudaLibrary_t l : k->libs)
    if (l) cudaLibraryUnload(l);
  k->libs.clear();
  k->kern.clear();
}

}  // namespace rtlsim
