// rx_codegen.cpp -- emits the CUDA C program bodies of each regex group
// (BitGen emits "optimized GPU kernels" source-to-source and compiles them
// with NVRTC, Sec. 3.1 / P:L380; here the emitted part is only the
// straight-line per-group program, the loop/prologue/epilogue template is the
// hand-written rx_device.cuh).
//
// Character classes (Fig. 2a) are emitted as a reduced ordered BDD
// over the basis streams, MSB (paper b0) first: every node is one mux /
// and / or / andnot, which ptxas packs into LOP3s.
#include <cstring>
#include <functional>
#include <map>
#include <sstream>

#include "rx_internal.h"

namespace rx {
namespace {

struct TabKey {
  int level;
  uint64_t w[4];
  bool operator<(const TabKey &o) const {
    if (level != o.level) return level < o.level;
    return std::memcmp(w, o.w, sizeof w) < 0;
  }
};

// truth table helpers: a table at `level` has 2^level meaningful bits
static bool tab_bit(const uint64_t *w, int i) { return (w[i >> 6] >> (i & 63)) & 1; }

struct RegexEmitter {
  std::ostringstream &os;
  const RegexIR &ir;
  int K;
  int rloc;        // member index in the group
  int slot_base;   // first state slot of this regex in the group
  std::vector<std::map<TabKey, std::string>> cc_scope;
  std::vector<std::map<std::vector<uint64_t>, std::string>> set_scope;
  int tmp = 0;
  std::string V;

  RegexEmitter(std::ostringstream &o, const RegexIR &r, int k, int rl, int sb)
      : os(o), ir(r), K(k), rloc(rl), slot_base(sb) {
    V = "V<" + std::to_string(K) + ">";
  }

  std::string ind(int n) { return std::string(2 * n, ' '); }
  std::string nv(int id) { return "n" + std::to_string(rloc) + "_" + std::to_string(id); }
  std::string fresh() { return "t" + std::to_string(rloc) + "_" + std::to_string(tmp++); }

  // --- character classes -------------------------------------------------
  std::string bdd(int level, const uint64_t *tab, int in) {
    int n = 1 << level;
    bool all0 = true, all1 = true;
    for (int i = 0; i < n; ++i) {
      if (tab_bit(tab, i)) all0 = false; else all1 = false;
    }
    if (all0) return "#0";
    if (all1) return "#1";
    TabKey key{level, {0, 0, 0, 0}};
    for (int i = 0; i < n; ++i)
      if (tab_bit(tab, i)) key.w[i >> 6] |= 1ull << (i & 63);
    for (auto it = cc_scope.rbegin(); it != cc_scope.rend(); ++it) {
      auto f = it->find(key);
      if (f != it->end()) return f->second;
    }
    int h = n / 2;
    uint64_t t0[4] = {0, 0, 0, 0}, t1[4] = {0, 0, 0, 0};
    for (int i = 0; i < h; ++i) {
      if (tab_bit(tab, i)) t0[i >> 6] |= 1ull << (i & 63);
      if (tab_bit(tab, i + h)) t1[i >> 6] |= 1ull << (i & 63);
    }
    std::string f0 = bdd(level - 1, t0, in), f1 = bdd(level - 1, t1, in);
    std::string b = "c.bit[" + std::to_string(level - 1) + "]";
    std::string e;
    if (f0 == f1) return f0;
    if (f0 == "#0" && f1 == "#1") e = b;
    else if (f0 == "#1" && f1 == "#0") e = "vnot(" + b + ")";
    else if (f0 == "#0") e = "vand(" + b + ", " + f1 + ")";
    else if (f1 == "#0") e = "vandn(" + f0 + ", " + b + ")";
    else if (f1 == "#1") e = "vor(" + b + ", " + f0 + ")";
    else if (f0 == "#1") e = "vornot(" + f1 + ", " + b + ")";
    else e = "vsel(" + b + ", " + f1 + ", " + f0 + ")";
    std::string t = fresh();
    os << ind(in) << "const " << V << " " << t << " = " << e << ";\n";
    cc_scope.back()[key] = t;
    return t;
  }

  std::string cc(const ByteSet &s, int in) {
    std::vector<uint64_t> k(s.w, s.w + 4);
    for (auto it = set_scope.rbegin(); it != set_scope.rend(); ++it) {
      auto f = it->find(k);
      if (f != it->end()) return f->second;
    }
    std::string e = bdd(8, s.w, in);
    std::string out;
    if (e == "#0") out = "vzero<" + std::to_string(K) + ">()";
    else if (e == "#1") out = "c.vm";
    else if (s.has(0)) {
      // a class containing 0x00 would match the zero padding: mask with the
      // valid-data stream (reading c9)
      out = fresh();
      os << ind(in) << "const " << V << " " << out << " = vand(" << e << ", c.vm);\n";
    } else {
      out = e;
    }
    set_scope.back()[k] = out;
    return out;
  }

  void push() { cc_scope.emplace_back(); set_scope.emplace_back(); }
  void pop() { cc_scope.pop_back(); set_scope.pop_back(); }

  // state slots read by stateful sites inside a block (for guard pending tests)
  void collect_slots(int block, std::vector<int> &out) {
    for (int id : ir.blocks[block].nodes) {
      const Node &n = ir.nodes[id];
      if (n.slot >= 0) out.push_back(n.slot);
      if (n.op == Op::Loop || n.op == Op::Guard) collect_slots(n.sub, out);
    }
  }

  std::string st(int slot) { return "st[" + std::to_string(slot_base + slot) + "]"; }
  std::string nst(int slot) { return "nst[" + std::to_string(slot_base + slot) + "]"; }

  void block(int b, int in, const std::string &first) {
    for (int id : ir.blocks[b].nodes) node(id, in, first);
  }

  void node(int id, int in, const std::string &first) {
    const Node &n = ir.nodes[id];
    std::string I = ind(in);
    auto A = [&] { return nv(n.a); };
    auto B = [&] { return nv(n.b); };
    switch (n.op) {
      case Op::Zero: os << I << "const " << V << " " << nv(id) << " = vzero<" << K << ">();\n"; break;
      case Op::Ones: os << I << "const " << V << " " << nv(id) << " = vones<" << K << ">();\n"; break;
      case Op::Fr: break;  // declared by the loop
      case Op::CC: {
        std::string e = cc(ir.sets[n.cc], in);
        os << I << "const " << V << " " << nv(id) << " = " << e << ";\n";
        break;
      }
      case Op::And: os << I << "const " << V << " " << nv(id) << " = vand(" << A() << ", " << B() << ");\n"; break;
      case Op::Or: os << I << "const " << V << " " << nv(id) << " = vor(" << A() << ", " << B() << ");\n"; break;
      case Op::Xor: os << I << "const " << V << " " << nv(id) << " = vxor(" << A() << ", " << B() << ");\n"; break;
      case Op::AndNot: os << I << "const " << V << " " << nv(id) << " = vandn(" << A() << ", " << B() << ");\n"; break;
      case Op::Adv:
        if (n.loop >= 0) {
          os << I << "const " << V << " " << nv(id) << " = advf(c, " << A() << ", " << n.aw << ", " << first
             << " ? " << st(n.slot) << " : 0u, " << nst(n.slot) << ");\n";
        } else {
          os << I << "const " << V << " " << nv(id) << " = vadv<" << n.k << ">(" << A() << ");\n";
        }
        break;
      case Op::Look: os << I << "const " << V << " " << nv(id) << " = vlook<" << n.k << ">(" << A() << ");\n"; break;
      case Op::MStar:
        if (n.loop >= 0) {
          std::string co = fresh();
          os << I << "u32 " << co << ";\n";
          os << I << "const " << V << " " << nv(id) << " = mstar(c, " << A() << ", " << B() << ", " << n.aw << ", "
             << first << " ? " << st(n.slot) << " : 0u, " << co << ");\n";
          os << I << nst(n.slot) << " |= " << co << ";\n";
        } else {
          os << I << "const " << V << " " << nv(id) << " = mstar(c, " << A() << ", " << B() << ", " << n.aw << ", "
             << st(n.slot) << ", " << nst(n.slot) << ");\n";
        }
        break;
      case Op::Loop: {
        // while-fixpoint of Fig. 2e / Listing 3
        std::string L = std::to_string(rloc) + "_" + std::to_string(id);
        std::string acc = "acc" + L, fr = "fr" + L, fst = "first" + L, it = "it" + L, nw = "nw" + L;
        os << I << V << " " << nv(id) << ";\n" << I << "{\n";
        // k=1: the operand holds ends of r (acc starts with them);
        // k=0: the operand holds prefix ends (the first frontier only)
        if (n.k == 1) {
          os << I << "  " << V << " " << acc << " = vmask_ge(c, " << A() << ", " << n.aw << ");\n";
          os << I << "  " << V << " " << fr << " = " << acc << ";\n";
        } else {
          os << I << "  " << V << " " << acc << " = vzero<" << K << ">();\n";
          os << I << "  " << V << " " << fr << " = vmask_ge(c, " << A() << ", " << n.aw << ");\n";
        }
        os << I << "  bool " << fst << " = " << (first.empty() ? "true" : first) << ";\n";
        os << I << "  u32 " << it << " = 0u;\n";
        os << I << "  while (true) {\n";
        os << I << "    const " << V << " " << nv(n.fr) << " = " << fr << ";\n";
        push();
        block(n.sub, in + 2, fst);
        pop();
        os << I << "    const " << V << " " << nw << " = vmask_ge(c, vandn(" << nv(n.res) << ", " << acc << "), "
           << n.aw << ");\n";
        os << I << "    if (!vany(" << nw << ")) break;\n";
        os << I << "    " << acc << " = vor(" << acc << ", " << nw << ");\n";
        os << I << "    " << fr << " = " << nw << ";\n";
        os << I << "    " << fst << " = false;\n";
        os << I << "    if (++" << it << " > RX_LOOP_CAP) { if (c.lane == 0) atomicOr(c.status, 1u); break; }\n";
        os << I << "  }\n";
        os << I << "  " << nv(id) << " = " << acc << ";\n";
        os << I << "}\n";
        break;
      }
      case Op::Guard: {
        // Zero Block Skipping (Sec. 6): skip the region when the
        // zero-path head is all-zero in the window and no state flows in.
        std::vector<int> slots;
        collect_slots(n.sub, slots);
        std::string pend;
        for (size_t i = 0; i < slots.size(); ++i) pend += (i ? " | " : "") + st(slots[i]);
        os << I << V << " " << nv(id) << " = vzero<" << K << ">();\n";
        os << I << "if (vany(" << A() << ")" << (pend.empty() ? "" : " || ((" + pend + ") != 0u)") << ") {\n";
        push();
        block(n.sub, in + 1, first);
        pop();
        os << I << "  " << nv(id) << " = " << nv(n.res) << ";\n";
        os << I << "}\n";
        break;
      }
    }
  }

  void emit_regex() {
    os << "    {  // regex member " << rloc << "\n";
    push();
    block(0, 3, "");
    pop();
    const Node &o = ir.nodes[ir.out];
    if (o.op != Op::Zero) os << "      emit(c, " << rloc << ", " << nv(ir.out) << ");\n";
    os << "    }\n";
  }
};

}  // namespace

extern const char *kDevicePrelude;

std::string emit_program_source_range(CompiledSet &cs, int g_begin, int g_end, uint32_t sbase0) {
  std::ostringstream os;
  os << kDevicePrelude << "\n// ===================== generated program =====================\n";
  int G = g_end - g_begin;
  int nsmax = 0, nrmax = 1, sbase = (int)sbase0;
  for (int gi = g_begin; gi < g_end; ++gi) {
    nsmax = std::max(nsmax, cs.groups[gi].nslots);
    nrmax = std::max(nrmax, (int)cs.groups[gi].regexes.size());
  }
  if (nsmax < 1) nsmax = 1;
  os << "#define RX_NG " << G << "\n#define RX_NSMAX " << nsmax << "\n#define RX_NRMAX " << nrmax << "\n";
  for (int gi = 0; gi < G; ++gi) {
    Group &g = cs.groups[g_begin + gi];
    os << "__device__ const int rx_rid_" << gi << "[" << g.regexes.size() << "] = {";
    for (size_t i = 0; i < g.regexes.size(); ++i) os << (i ? "," : "") << g.regexes[i];
    os << "};\n";
    os << "struct RxG" << gi << " {\n";
    os << "  static constexpr int K = " << g.K << ", Lw = " << g.Lw << ", Bw = " << g.Bw << ", NS = " << g.nslots
       << ", NR = " << g.regexes.size() << ", SBASE = " << sbase << ", NG = " << G << ", GID = " << gi
       << ", NSMAX = " << nsmax << ";\n";
    os << "  static DEV const int *rid() { return rx_rid_" << gi << "; }\n";
    os << "  static DEV void body(Ctx<" << g.K << "> &c, const u32 *st, u32 *nst) {\n";
    os << "    (void)st; (void)nst;\n";
    for (size_t m = 0; m < g.regexes.size(); ++m) {
      RegexEmitter em(os, cs.irs[g.regexes[m]], g.K, (int)m, g.slot_base[m]);
      em.emit_regex();
    }
    os << "  }\n};\n";
    // one non-inlined function per group and pass: ptxas compiles each
    // separately (compile time stays linear in the number of groups)
    os << "__device__ __noinline__ void rx_seg_" << gi << "(const RxParams &p, int seg, u64 *acc) { rx_run_segment<RxG"
       << gi << ">(p, seg, acc); }\n";
    if (g.nslots > 0)
      os << "__device__ __noinline__ void rx_fix_" << gi << "(const RxParams &p, u64 *acc) { rx_fixup_group<RxG" << gi
         << ">(p, acc); }\n";
    sbase += g.nslots;
  }
  os << "\nextern \"C\" __global__ void __launch_bounds__(128) rx_pass1(const RxParams p) {\n"
        "  extern __shared__ u64 rx_smem[];\n"
        "  const int warp = threadIdx.x >> 5;\n"
        "  u64 *acc = rx_smem + warp * (3 * RX_NRMAX);\n"
        "  const long long wid = (long long)blockIdx.x * (blockDim.x >> 5) + warp;\n"
        "  const int g = (int)(wid % RX_NG);\n"
        "  const long long seg = wid / RX_NG;\n"
        "  if (seg >= p.nseg_max) return;\n"
        "  switch (g) {\n";
  for (int gi = 0; gi < G; ++gi) os << "    case " << gi << ": rx_seg_" << gi << "(p, (int)seg, acc); break;\n";
  os << "    default: break;\n  }\n}\n";
  os << "\nextern \"C\" __global__ void __launch_bounds__(128) rx_fixup(const RxParams p) {\n"
        "  extern __shared__ u64 rx_smem[];\n"
        "  const int warp = threadIdx.x >> 5;\n"
        "  u64 *acc = rx_smem + warp * (3 * RX_NRMAX);\n"
        "  const long long g = (long long)blockIdx.x * (blockDim.x >> 5) + warp;\n"
        "  if (g >= RX_NG) return;\n"
        "  switch ((int)g) {\n";
  for (int gi = 0; gi < G; ++gi)
    if (cs.groups[g_begin + gi].nslots > 0) os << "    case " << gi << ": rx_fix_" << gi << "(p, acc); break;\n";
  os << "    default: break;\n  }\n}\n";
  return os.str();
}

}  // namespace rx
