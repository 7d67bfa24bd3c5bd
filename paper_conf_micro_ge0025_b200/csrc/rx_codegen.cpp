// rx_codegen.cpp -- emits the CUDA C program bodies of each regex group
// (BitGen emits "optimized GPU kernels" source-to-source and compiles them
// with NVRTC, Sec. 3.1 / P:L380; here the emitted part is only the
// straight-line per-group program, the loop/prologue/epilogue template is the
// hand-written rx_device.cuh).
//
// The emitted code is flat per-word scalar C (u32 variables, intrinsics):
// each IR value of K words per lane becomes K registers; NVVM compiles flat
// code an order of magnitude faster than template-per-op code.
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

static bool tab_bit(const uint64_t *w, int i) { return (w[i >> 6] >> (i & 63)) & 1; }

struct RegexEmitter {
  std::ostringstream &os;
  const RegexIR &ir;
  int K;
  int rloc;       // cluster index in the group (names)
  int slot_base;  // first state slot of this regex in the group
  // CC / BDD-node caches by scope; scope 0 is shared by all regexes of the
  // group (their unguarded heads), deeper scopes are guard / loop bodies
  std::vector<std::map<TabKey, std::string>> &cc_scope;
  std::vector<std::map<std::vector<uint64_t>, std::string>> &set_scope;
  int tmp = 0;
  std::string lit_pool;          // name of the group's literal byte table
  std::vector<int> lit_off;      // offset of ir.lits[i] in it

  RegexEmitter(std::ostringstream &o, const RegexIR &r, int k, int rl, int sb,
               std::vector<std::map<TabKey, std::string>> &ccs,
               std::vector<std::map<std::vector<uint64_t>, std::string>> &sets)
      : os(o), ir(r), K(k), rloc(rl), slot_base(sb), cc_scope(ccs), set_scope(sets) {}

  std::string ind(int n) { return std::string(2 * n, ' '); }
  std::string nv(int id) { return "n" + std::to_string(rloc) + "_" + std::to_string(id); }
  std::string fresh() { return "t" + std::to_string(rloc) + "_" + std::to_string(tmp++); }
  // word i of a vector value; "#0" / "#1" are the constant streams
  std::string W(const std::string &b, int i) {
    if (b == "#0") return "0u";
    if (b == "#1") return "0xffffffffu";
    return b + "w" + std::to_string(i);
  }
  std::string widx(int i) { return "(int)(" + std::to_string(K) + "u * lane + " + std::to_string(i) + "u)"; }

  void decl(int in, const std::string &dst, const std::function<std::string(int)> &e, bool cst = true) {
    for (int i = 0; i < K; ++i) os << ind(in) << (cst ? "const u32 " : "u32 ") << W(dst, i) << " = " << e(i) << ";\n";
  }
  void assign(int in, const std::string &dst, const std::function<std::string(int)> &e) {
    for (int i = 0; i < K; ++i) os << ind(in) << W(dst, i) << " = " << e(i) << ";\n";
  }
  std::string any(const std::string &b) {
    std::string o;
    for (int i = 0; i < K; ++i) o += (i ? " | " : "") + W(b, i);
    return "__any_sync(RX_FULL, (" + o + ") != 0u)";
  }
  // word (global index - q) of b, for word i of this lane
  std::string up(const std::string &b, int q, int i) {
    int src = i - q;
    if (src >= 0) return W(b, src);
    int d = (-src + K - 1) / K;
    int reg = ((src % K) + K) % K;
    return "__shfl_up_sync(RX_FULL, " + W(b, reg) + ", " + std::to_string(d) + ")";
  }
  std::string down(const std::string &b, int q, int i) {
    int src = i + q;
    int d = src / K, reg = src % K;
    if (d == 0) return W(b, reg);
    return "__shfl_down_sync(RX_FULL, " + W(b, reg) + ", " + std::to_string(d) + ")";
  }
  // Advance (paper "S >> n"): out[p] = in[p - n]
  void adv(int in, const std::string &dst, const std::string &a, int n) {
    int Q = n / 32, R = n % 32;
    if (R == 0) {
      decl(in, dst, [&](int i) { return up(a, Q, i); });
      return;
    }
    decl(in, dst, [&](int i) {
      return "__funnelshift_l(" + up(a, Q + 1, i) + ", " + up(a, Q, i) + ", " + std::to_string(R) + ")";
    });
  }
  // Lookahead (paper "S << n"): out[p] = in[p + n]
  void look(int in, const std::string &dst, const std::string &a, int n) {
    int Q = n / 32, R = n % 32;
    if (R == 0) {
      decl(in, dst, [&](int i) { return down(a, Q, i); });
      return;
    }
    decl(in, dst, [&](int i) {
      return "__funnelshift_r(" + down(a, Q, i) + ", " + down(a, Q + 1, i) + ", " + std::to_string(R) + ")";
    });
  }
  // broadcast of word `wexpr` (runtime) of b
  std::string extract(const std::string &b, const std::string &wexpr) {
    if (K == 1) return "__shfl_sync(RX_FULL, " + W(b, 0) + ", " + wexpr + ")";
    std::string sel = W(b, K - 1);
    for (int i = K - 2; i >= 0; --i)
      sel = "((" + wexpr + ") % " + std::to_string(K) + " == " + std::to_string(i) + " ? " + W(b, i) + " : " + sel + ")";
    return "__shfl_sync(RX_FULL, " + sel + ", (" + wexpr + ") / " + std::to_string(K) + ")";
  }

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
    if (f0 == f1) return f0;
    std::string b = "b" + std::to_string(level - 1);
    std::string t = fresh();
    decl(in, t, [&](int i) {
      std::string B = W(b, i), F0 = W(f0, i), F1 = W(f1, i);
      if (f0 == "#0" && f1 == "#1") return B;
      if (f0 == "#1" && f1 == "#0") return "~" + B;
      if (f0 == "#0") return "(" + B + " & " + F1 + ")";
      if (f1 == "#0") return "(" + F0 + " & ~" + B + ")";
      if (f1 == "#1") return "(" + B + " | " + F0 + ")";
      if (f0 == "#1") return "(" + F1 + " | ~" + B + ")";
      return "((" + B + " & " + F1 + ") | (~" + B + " & " + F0 + "))";
    });
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
    if (e == "#0") out = "#0";
    else if (e == "#1") out = "vm";
    else if (s.has(0)) {
      // a class containing 0x00 would match the zero padding: mask with the
      // valid-data stream (reading c9)
      out = fresh();
      decl(in, out, [&](int i) { return W(e, i) + " & " + W("vm", i); });
    } else {
      out = e;
    }
    set_scope.back()[k] = out;
    return out;
  }

  void push() { cc_scope.emplace_back(); set_scope.emplace_back(); }
  void pop() { cc_scope.pop_back(); set_scope.pop_back(); }

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

  // MatchStar in match-end form: ((((X + C) ^ C) | X) & C), X masked to
  // words >= aw; long add = per-lane K-word add + generate/propagate ballots
  // + carry-lookahead on lane masks; carry in at word aw, carry into word
  // aw+cw out.
  void mstar(int in, const std::string &dst, const std::string &X, const std::string &C, int aw,
             const std::string &cin, const std::string &cout_lhs, bool accumulate) {
    std::string p = fresh();
    std::string I = ind(in);
    decl(in, dst, [&](int) { return std::string("0u"); }, false);
    os << I << "{\n";
    std::string J = ind(in + 1);
    for (int i = 0; i < K; ++i)
      os << J << "const u32 " << p << "x" << i << " = " << widx(i) << " >= " << aw << " ? " << W(X, i) << " : 0u;\n";
    os << J << "u32 " << p << "c = 0u; bool " << p << "p = true;\n";
    for (int i = 0; i < K; ++i) {
      os << J << "u32 " << p << "s" << i << ";\n";
      os << J << "{ const unsigned long long t = (unsigned long long)" << p << "x" << i << " + " << W(C, i) << " + ("
         << widx(i) << " == " << aw << " ? (" << cin << ") : 0u) + " << p << "c; " << p << "s" << i
         << " = (u32)t; " << p << "c = (u32)(t >> 32); " << p << "p = " << p << "p && (" << p << "s" << i
         << " == 0xffffffffu); }\n";
    }
    os << J << "const u32 " << p << "G = __ballot_sync(RX_FULL, " << p << "c != 0u);\n";
    os << J << "const u32 " << p << "P = __ballot_sync(RX_FULL, " << p << "p);\n";
    os << J << "const u32 " << p << "A = " << p << "G | " << p << "P;\n";
    os << J << "const u32 " << p << "v = (" << p << "A + " << p << "G) ^ " << p << "A ^ " << p << "G;\n";
    os << J << "u32 " << p << "l = (" << p << "v >> lane) & 1u;\n";
    for (int i = 0; i < K; ++i) {
      os << J << "{ const unsigned long long t = (unsigned long long)" << p << "s" << i << " + " << p << "l; " << p
         << "s" << i << " = (u32)t; " << p << "l = (u32)(t >> 32); }\n";
      os << J << W(dst, i) << " = ((" << p << "s" << i << " ^ " << W(C, i) << ") | " << p << "x" << i << ") & "
         << W(C, i) << ";\n";
      os << J << "const u32 " << p << "qw" << i << " = " << p << "s" << i << " ^ " << p << "x" << i << " ^ "
         << W(C, i) << ";\n";
    }
    os << J << "const int " << p << "e = " << aw << " + cw;\n";
    os << J << "const u32 " << p << "top = (" << p << "G >> 31) | ((" << p << "P >> 31) & (" << p << "v >> 31) & 1u);\n";
    os << J << "const u32 " << p << "in = "
       << extract(p + "q", "(" + p + "e < " + std::to_string(32 * K) + " ? " + p + "e : 0)") << " & 1u;\n";
    os << J << cout_lhs << (accumulate ? " |= " : " = ") << "(" << p << "e >= " << 32 * K << " ? " << p << "top : " << p
       << "in);\n";
    os << I << "}\n";
  }

  void node(int id, int in, const std::string &first) {
    const Node &n = ir.nodes[id];
    std::string I = ind(in);
    auto val = [&](int x) -> std::string {  // Zero / Ones operands fold to constants
      if (x < 0) return "";
      if (ir.nodes[x].op == Op::Zero) return "#0";
      if (ir.nodes[x].op == Op::Ones) return "#1";
      return nv(x);
    };
    std::string A = val(n.a), B = val(n.b);
    switch (n.op) {
      case Op::Zero: case Op::Ones: case Op::Fr: break;
      case Op::CC: {
        std::string e = cc(ir.sets[n.cc], in);
        decl(in, nv(id), [&](int i) { return W(e, i); });
        break;
      }
      case Op::And: decl(in, nv(id), [&](int i) { return W(A, i) + " & " + W(B, i); }); break;
      case Op::Or: decl(in, nv(id), [&](int i) { return W(A, i) + " | " + W(B, i); }); break;
      case Op::Xor: decl(in, nv(id), [&](int i) { return W(A, i) + " ^ " + W(B, i); }); break;
      case Op::AndNot: decl(in, nv(id), [&](int i) { return W(A, i) + " & ~" + W(B, i); }); break;
      case Op::Adv:
        if (n.loop >= 0) {
          // forwarded advance inside a loop body: inject the previous
          // window's operand word at aw-1 (first iteration only), collect
          // the word at aw-1+cw for the next window
          std::string t = fresh();
          decl(in, t, [&](int i) {
            return W(A, i) + " | (" + widx(i) + " == " + std::to_string(n.aw - 1) + " && " + first + " ? " + st(n.slot) +
                   " : 0u)";
          });
          os << I << nst(n.slot) << " |= " << extract(t, std::to_string(n.aw - 1) + " + cw") << ";\n";
          adv(in, nv(id), t, n.k);
        } else {
          adv(in, nv(id), A, n.k);
        }
        break;
      case Op::Look: look(in, nv(id), A, n.k); break;
      case Op::Lit: {
        // literal run confirmed byte by byte at the (sparse) marker bits
        std::string t = fresh();
        os << I << "V<" << K << "> " << t << "i;\n";
        for (int i = 0; i < K; ++i) os << I << t << "i.w[" << i << "] = " << W(A, i) << ";\n";
        os << I << "const V<" << K << "> " << t << "o = rx_lit<" << K << ">(c.lane, rx_smem_addr(c.wb), rx_smem_addr(c.ob), " << t << "i, " << lit_pool << " + "
           << lit_off[n.cc] << ", " << n.k << ");\n";
        decl(in, nv(id), [&](int i) { return t + "o.w[" + std::to_string(i) + "]"; });
        break;
      }
      case Op::MStar:
        if (n.loop >= 0)
          mstar(in, nv(id), A, B, n.aw, "(" + first + " ? " + st(n.slot) + " : 0u)", nst(n.slot), true);
        else
          mstar(in, nv(id), A, B, n.aw, st(n.slot), nst(n.slot), false);
        break;
      case Op::Loop: {
        // while-fixpoint of Fig. 2e / Listing 3
        std::string L = std::to_string(rloc) + "_" + std::to_string(id);
        std::string acc = "acc" + L, fr = "fr" + L, fst = "first" + L, it = "it" + L, nw = "nw" + L;
        std::string aw = std::to_string(n.aw);
        decl(in, nv(id), [&](int) { return std::string("0u"); }, false);
        os << I << "{\n";
        // k=1: the operand holds ends of r (acc starts with them);
        // k=0: the operand holds prefix ends (the first frontier only)
        if (n.k == 1) {
          decl(in + 1, acc, [&](int i) { return widx(i) + " >= " + aw + " ? " + W(A, i) + " : 0u"; }, false);
          decl(in + 1, fr, [&](int i) { return W(acc, i); }, false);
        } else {
          decl(in + 1, acc, [&](int) { return std::string("0u"); }, false);
          decl(in + 1, fr, [&](int i) { return widx(i) + " >= " + aw + " ? " + W(A, i) + " : 0u"; }, false);
        }
        os << I << "  bool " << fst << " = " << (first.empty() ? "true" : first) << ";\n";
        os << I << "  u32 " << it << " = 0u;\n";
        os << I << "  while (true) {\n";
        decl(in + 2, nv(n.fr), [&](int i) { return W(fr, i); });
        push();
        block(n.sub, in + 2, fst);
        pop();
        std::string R = val(n.res);
        decl(in + 2, nw, [&](int i) { return widx(i) + " >= " + aw + " ? (" + W(R, i) + " & ~" + W(acc, i) + ") : 0u"; });
        os << I << "    if (!" << any(nw) << ") break;\n";
        assign(in + 2, acc, [&](int i) { return W(acc, i) + " | " + W(nw, i); });
        assign(in + 2, fr, [&](int i) { return W(nw, i); });
        os << I << "    " << fst << " = false;\n";
        os << I << "    if (++" << it << " > RX_LOOP_CAP) { if (lane == 0) atomicOr(c.o->status, 1u); break; }\n";
        os << I << "  }\n";
        assign(in + 1, nv(id), [&](int i) { return W(acc, i); });
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
        decl(in, nv(id), [&](int) { return std::string("0u"); }, false);
        os << I << "if (" << any(A) << (pend.empty() ? "" : " || ((" + pend + ") != 0u)") << ") {\n";
        push();
        block(n.sub, in + 1, first);
        pop();
        std::string R = val(n.res);
        assign(in + 1, nv(id), [&](int i) { return W(R, i); });
        os << I << "}\n";
        break;
      }
    }
  }

  std::vector<int> out_member;  // group member index of each IR output

  void emit_output(int in) {
    for (size_t k = 0; k < ir.outs.size(); ++k) {
      const Node &o = ir.nodes[ir.outs[k]];
      if (o.op == Op::Zero) continue;
      std::string I = ind(in);
      std::string R = nv(ir.outs[k]);
      std::string m;
      for (int i = 0; i < K; ++i) m += (i ? " | " : "") + ("(" + W(R, i) + " & c.cm[" + std::to_string(i) + "])");
      // walk-back runs (mode B) only compute state
      os << I << "if (!c.walk && (c.dense || __any_sync(RX_FULL, (" << m << ") != 0u))) {\n";
      // counts only: the popcount goes straight into the warp's shared
      // accumulator (REDUX), no out-of-line call
      os << I << "  if (c.fast) {\n" << I << "    const u32 cnt_ = __reduce_add_sync(RX_FULL, ";
      for (int i = 0; i < K; ++i) os << (i ? " + " : "") << "__popc(" << W(R, i) << " & c.cm[" << i << "])";
      os << ");\n" << I << "    if (lane == 0u) c.acc[" << 3 * out_member[k] << "] += (u64)cnt_;\n" << I << "  } else {\n";
      os << I << "  V<" << K << "> ov;\n";
      os << I << "  u32 cwb = 0u;\n";
      for (int i = 0; i < K; ++i) {
        os << I << "  ov.w[" << i << "] = " << W(R, i) << " & c.cm[" << i << "];\n";
        os << I << "  cwb |= (c.cm[" << i << "] != 0u ? 1u : 0u) << " << i << ";\n";
      }
      os << I << "  rx_emit<" << K << ">(c.o, " << out_member[k] << ", c.lane, c.word0, ov, cwb);\n";
      os << I << "  }\n" << I << "}\n";
    }
  }

  // Two-phase emission: phase 1 holds every
  // regex's unguarded head and the tests of its top-level zero-block guards,
  // contiguous in the instruction stream; phase 2 holds the guarded bodies,
  // the values depending on them and the output, and runs only for regexes
  // whose guard fired (or that carry state through such values).
  std::vector<char> post;   // top-level node depends on a guard result
  bool has_guard = false, stateful_post = false;

  void classify() {
    post.assign(ir.nodes.size(), 0);
    for (int id : ir.blocks[0].nodes) {
      const Node &n = ir.nodes[id];
      bool p = n.op == Op::Guard;
      if (n.a >= 0 && post[n.a]) p = true;
      if (n.b >= 0 && post[n.b]) p = true;
      post[id] = p;
      if (n.op == Op::Guard) has_guard = true;
      if (p && (n.op == Op::MStar || n.op == Op::Loop)) stateful_post = true;
    }
  }

  std::string fire(int id) { return "f" + std::to_string(rloc) + "_" + std::to_string(id); }

  // is top-level value `id` zero whenever no top-level guard fires (and no
  // state flows in)?
  bool zero_when_unfired(int id) {
    const Node &n = ir.nodes[id];
    switch (n.op) {
      case Op::Guard: case Op::Zero: return true;
      case Op::Ones: case Op::CC: case Op::Fr: return false;
      case Op::And: return zero_when_unfired(n.a) || zero_when_unfired(n.b);
      case Op::Or: case Op::Xor: return zero_when_unfired(n.a) && zero_when_unfired(n.b);
      case Op::AndNot: case Op::Adv: case Op::Look: case Op::MStar: case Op::Loop: case Op::Lit:
        return zero_when_unfired(n.a);
    }
    return false;
  }

  // phase 1: returns the C expression "this regex needs phase 2"
  std::string emit_phase1() {
    classify();
    os << "    // ---- cluster " << rloc << " (phase 1: unguarded head, guard tests)\n";
    std::string need;
    for (int id : ir.blocks[0].nodes) {
      const Node &n = ir.nodes[id];
      if (!post[id]) {
        node(id, 2, "");
        continue;
      }
      if (n.op == Op::Guard) {
        std::vector<int> slots;
        collect_slots(n.sub, slots);
        std::string pend;
        for (size_t i = 0; i < slots.size(); ++i) pend += (i ? " | " : "") + st(slots[i]);
        if (post[n.a]) {
          // a guard whose head depends on an earlier guard's result is tested
          // inline in phase 2; phase 2 must run if state flows into it
          if (!pend.empty()) need += (need.empty() ? "" : " || ") + ("((" + pend + ") != 0u)");
          continue;
        }
        std::string cond = ir.nodes[n.a].op == Op::Ones ? "true" : any(nv(n.a));
        decl(2, nv(id), [&](int) { return std::string("0u"); }, false);
        os << "    const bool " << fire(id) << " = " << cond << (pend.empty() ? "" : " || ((" + pend + ") != 0u)")
           << ";\n";
        need += (need.empty() ? "" : " || ") + fire(id);
      }
    }
    if (!has_guard) emit_output(2);
    if (stateful_post) return "true";
    // the output must be produced even when no guard fires if it has an
    // unguarded contribution (e.g. an alternation with an unguarded branch)
    if (has_guard)
      for (int o : ir.outs)
        if (!zero_when_unfired(o)) return "true";
    return has_guard ? need : "";
  }

  // phase 2 (inside `if (need)`)
  void emit_phase2() {
    if (!has_guard) return;
    os << "    // ---- cluster " << rloc << " (phase 2: guarded bodies)\n";
    push();
    for (int id : ir.blocks[0].nodes) {
      if (!post[id]) continue;
      const Node &n = ir.nodes[id];
      if (n.op == Op::Guard && post[n.a]) {
        node(id, 2, "");  // inline guard (head computed in phase 2)
      } else if (n.op == Op::Guard) {
        os << "    if (" << fire(id) << ") {\n";
        push();
        block(n.sub, 3, "");
        pop();
        std::string R = ir.nodes[n.res].op == Op::Zero ? "#0" : nv(n.res);
        assign(3, nv(id), [&](int i) { return W(R, i); });
        os << "    }\n";
      } else {
        node(id, 2, "");
      }
    }
    emit_output(2);
    pop();
  }
};

}  // namespace

extern const char *kDevicePrelude;

static void layout(const CompiledSet &cs, int &nsmax, int &nrmax) {
  nsmax = 1;
  nrmax = 1;
  for (auto &g : cs.groups) {
    nsmax = std::max(nsmax, g.nslots);
    nrmax = std::max(nrmax, (int)g.regexes.size());
  }
}
// per-warp shared bytes of the literal-run scratch (frame bytes + output words)
int lit_scratch_bytes(const CompiledSet &cs) {
  int kmax = 1;
  bool any = false;
  for (auto &g : cs.groups) {
    kmax = std::max(kmax, g.K);
    for (auto &c : g.clusters) any = any || !c.ir.lits.empty();
  }
  return any ? 1152 * kmax : 0;
}
int max_words_per_lane(const CompiledSet &cs) {
  int kmax = 1;
  for (auto &g : cs.groups) kmax = std::max(kmax, g.K);
  return kmax;
}

// One relocatable compilation unit per group (NVRTC -rdc): the group's
// traits, its program body, and the two non-inlined entry functions
// rx_seg_<g> (pass 1 over one segment) and rx_fix_<g> (carry fix-up).
// Compile time stays linear in the number of groups; the CUDA driver links
// the units with the kernel unit into one module.
std::string emit_group_unit(CompiledSet &cs, int gi) {
  std::ostringstream os;
  os << kDevicePrelude << "\n// ===================== generated group " << gi << " =====================\n";
  int nsmax, nrmax;
  layout(cs, nsmax, nrmax);
  int G = (int)cs.groups.size();
  int sbase = 0;
  for (int h = 0; h < gi; ++h) sbase += cs.groups[h].nslots;
  Group &g = cs.groups[gi];
  // the group's literal runs (Op::Lit), one byte table
  std::vector<std::vector<int>> lit_off(g.clusters.size());
  std::string pool;
  for (size_t ci = 0; ci < g.clusters.size(); ++ci)
    for (auto &l : g.clusters[ci].ir.lits) {
      lit_off[ci].push_back((int)pool.size());
      pool += l;
    }
  os << "__device__ const unsigned char rx_litb_" << gi << "[" << std::max<size_t>(pool.size(), 1) << "] = {";
  for (size_t i = 0; i < pool.size(); ++i) os << (i ? "," : "") << (unsigned)(unsigned char)pool[i];
  if (pool.empty()) os << "0";
  os << "};\n";
  os << "__device__ const int rx_rid_" << gi << "[" << g.regexes.size() << "] = {";
  for (size_t i = 0; i < g.regexes.size(); ++i) os << (i ? "," : "") << g.regexes[i];
  os << "};\n";
  const int NC = (int)g.clusters.size();
  std::vector<uint32_t> cmask(NC, 0u);
  for (int ci = 0; ci < NC; ++ci)
    for (int m : g.clusters[ci].members) cmask[ci] |= 1u << m;
  // per state slot: its cluster, and its top value (the largest state it can
  // hold: a MatchStar carry is 0/1, a forwarded advance tail a whole word)
  // for the mode-B walk-back
  std::vector<uint32_t> sci(std::max(g.nslots, 1), 0u), top(std::max(g.nslots, 1), 0u);
  uint32_t calways = 0u, cbcap = 0u;
  for (int ci = 0; ci < NC; ++ci) {
    const Cluster &cl = g.clusters[ci];
    if (cl.always) calways |= 1u << ci;
    if (cl.bcap) cbcap |= 1u << ci;
    for (auto &n : cl.ir.nodes)
      if (n.slot >= 0) {
        sci[cl.slot_base + n.slot] = (uint32_t)ci;
        top[cl.slot_base + n.slot] = n.op == Op::MStar ? 1u : 0xffffffffu;
      }
  }
  os << "__device__ const unsigned char rx_sci_" << gi << "[" << sci.size() << "] = {";
  for (size_t i = 0; i < sci.size(); ++i) os << (i ? "," : "") << sci[i];
  os << "};\n__device__ const unsigned rx_top_" << gi << "[" << top.size() << "] = {";
  for (size_t i = 0; i < top.size(); ++i) os << (i ? "," : "") << top[i] << "u";
  os << "};\n__device__ const unsigned rx_cm_" << gi << "[" << std::max(NC, 1) << "] = {";
  for (int ci = 0; ci < NC; ++ci) os << (ci ? "," : "") << cmask[ci] << "u";
  if (NC == 0) os << "0u";
  os << "};\n";
  os << "struct RxG" << gi << " {\n";
  os << "  static constexpr int K = " << g.K << ", Lw = " << g.Lw << ", Bw = " << g.Bw << ", NS = " << g.nslots
     << ", NR = " << g.regexes.size() << ", SBASE = " << sbase << ", NG = " << G << ", GID = " << gi
     << ", NSMAX = " << nsmax << ", NC = " << NC << ";\n";
  os << "  static DEV const int *rid() { return rx_rid_" << gi << "; }\n";
  os << "  static constexpr unsigned ALWAYS = " << g.always << "u;    // members without a first factor\n";
  os << "  static constexpr unsigned CALWAYS = " << calways << "u;   // clusters of them\n";
  os << "  static constexpr unsigned CBCAP = " << cbcap << "u;     // clusters that may run output-gated\n";
  os << "  static constexpr bool PF = " << (cs.use_pf ? "true" : "false") << ";\n";
  os << "  static constexpr bool LIT = " << (pool.empty() ? "false" : "true") << ";\n";
  os << "  static DEV u32 sci(int s) { return (u32)__ldg(&rx_sci_" << gi << "[s]); }\n";
  os << "  static DEV u32 top(int s) { return __ldg(&rx_top_" << gi << "[s]); }\n";
  os << "  static DEV u32 cmask(int ci) { return __ldg(&rx_cm_" << gi << "[ci]); }\n";
  // The group's program: one block of code per factor cluster, entered only
  // for the clusters in `run` (a cluster bitmask computed by the runner:
  // prefilter hits, carried state, walk-back targets) -- the warp jumps from
  // one active cluster to the next instead of walking past the inactive
  // ones.  body() is the out-of-line copy shared by the walk-back and both
  // fix-up runs; body_i is inlined into pass 1's sparse runner (the basis
  // planes and the window context stay in registers).
  auto emit_fn = [&](const std::string &name, bool inl) {
    os << "  static __device__ " << (inl ? "__forceinline__" : "__noinline__") << " void " << name << "(Ctx<" << g.K
       << "> &c, const u32 (&pl)[8][" << g.K << "], const u32 *st, u32 *nst, u32 run) {\n";
    os << "    (void)st; (void)nst;\n";
    os << "    const u32 lane = c.lane; const int cw = (int)c.cw; (void)cw; (void)lane;\n";
    for (int k = 0; k < 8; ++k)
      for (int i = 0; i < g.K; ++i)
        os << "    const u32 b" << k << "w" << i << " = pl[" << k << "][" << i << "]; (void)b" << k << "w" << i << ";\n";
    for (int i = 0; i < g.K; ++i) os << "    const u32 vmw" << i << " = c.vm[" << i << "]; (void)vmw" << i << ";\n";
    os << "    while (run) {\n      const int ci = __ffs(run) - 1;\n      run &= run - 1u;\n      switch (ci) {\n";
    for (int ci = 0; ci < NC; ++ci) {
      const Cluster &cl = g.clusters[ci];
      std::vector<std::map<TabKey, std::string>> ccs(1);
      std::vector<std::map<std::vector<uint64_t>, std::string>> sets(1);
      RegexEmitter em(os, cl.ir, g.K, ci, cl.slot_base, ccs, sets);
      em.out_member = cl.members;
      em.lit_pool = "rx_litb_" + std::to_string(gi);
      em.lit_off = lit_off[ci];
      // its unguarded (shared) head and guard tests (phase 1), then its
      // guarded bodies (phase 2) if a guard fired
      os << "      case " << ci << ": {\n";
      em.push();
      std::string need = em.emit_phase1();
      if (!need.empty()) {
        os << "    if (" << need << ") {\n";
        em.emit_phase2();
        os << "    }\n";
      }
      em.pop();
      os << "      } break;\n";
    }
    os << "      default: break;\n      }\n    }\n  }\n";
  };
  emit_fn("body", false);
  emit_fn("body_i", true);
  os << "};\n";
  // shared memory per warp (rx_runtime.cpp launch() mirrors it):
  //   acc [3*NRMAX] u64 | RxOut | state [6*NSMAX] u32 | literal-run scratch [LB]
  //   | window staging [TB] (TMA) | mbarrier u64
  const int LB = lit_scratch_bytes(cs), TB = 1024 * max_words_per_lane(cs);
  const int ACC = (24 * nrmax + 15) & ~15, OUTB = 96, STB = ((24 * nsmax) + 15) & ~15;
  const int PER = ACC + OUTB + STB + LB + TB + 16 + 512;  // + per-warp parameter copy (rx_match_batch)
  os << "static_assert(sizeof(RxOut) <= " << OUTB << ", \"RxOut layout\");\n";
  os << "#define RX_WARP_SMEM_" << gi << " " << PER << "\n";
  // The launch parameters are read from the CTA header of the dynamic shared
  // memory (rx_cta_params, copied there by the kernel): a reference to the
  // kernel parameter handed across this out-of-line call made every field
  // read a generic load through a spilled pointer (profiles/r2_*).
  os << "extern \"C\" __device__ __noinline__ void rx_seg_" << gi << "(int seg_in) {\n"
     << "  const RxParams &pc = rx_cta_params();\n"
     << "  const int warp = threadIdx.x >> 5;\n"
     << "  unsigned char *base = rx_warp_smem(warp, " << PER << ");\n"
     << "  RxParams *wp = reinterpret_cast<RxParams *>(base + " << PER - 512 << ");\n"
     << "  const bool batch = pc.batch_off != nullptr;\n"
     << "  u64 *acc = reinterpret_cast<u64 *>(base);\n"
     << "  RxOut *o = reinterpret_cast<RxOut *>(base + " << ACC << ");\n"
     << "  u32 *st = reinterpret_cast<u32 *>(base + " << ACC + OUTB << ");\n"
     << "  unsigned char *lb = base + " << ACC + OUTB + STB << ";\n"
     << "  unsigned char *tb = base + " << ACC + OUTB + STB + LB << ";\n"
     << "  u64 *bar = reinterpret_cast<u64 *>(base + " << ACC + OUTB + STB + LB + TB << ");\n"
     << "  (void)tb; (void)bar;\n"
     << "  // one run (a segment of the input), or one run per stream of this\n"
     << "  // warp's batch segment (one call site of the inlined runner)\n"
     << "  const long long nrun = batch ? pc.batch_spw : 1;\n"
     << "  for (long long k = 0; k < nrun; ++k) {\n"
     << "    const RxParams &p = batch ? rx_batch_view(pc, wp, (long long)seg_in * nrun + k, "
     << (int)cs.irs.size() << ") : pc;\n"
     << "    const int seg = batch ? 0 : seg_in;\n"
     << "    if (batch && !__syncthreads_or(!rx_batch_skip<RxG" << gi << ">(p, wp))) continue;\n";
  if (cs.use_pf)
    os << "    if (p.pf_on) { rx_run_segment_pf<RxG" << gi << ">(p, seg, o, acc, st, tb, bar, lb); continue; }\n";
  os << "    rx_run_segment_dense<RxG" << gi << ">(p, seg, o, acc, st, lb);\n  }\n}\n";
  if (g.nslots > 0)
    os << "extern \"C\" __device__ __noinline__ void rx_fix_" << gi << "(int seg) {\n"
       << "  const RxParams &p = rx_cta_params();\n"
       << "  const int warp = threadIdx.x >> 5;\n"
       << "  unsigned char *base = rx_warp_smem(warp, " << PER << ");\n"
       << "  rx_fixup_group<RxG" << gi << ">(p, reinterpret_cast<RxOut *>(base + " << ACC
       << "), reinterpret_cast<u64 *>(base), reinterpret_cast<u32 *>(base + " << ACC + OUTB << "), base + "
       << ACC + OUTB + STB << ", seg);\n}\n";
  return os.str();
}

// per-warp shared bytes of pass 1 / fix-up (must match emit_group_unit)
size_t warp_smem_bytes(const CompiledSet &cs) {
  int nsmax, nrmax;
  layout(cs, nsmax, nrmax);
  const int LB = lit_scratch_bytes(cs), TB = 1024 * max_words_per_lane(cs);
  return (size_t)(((24 * nrmax + 15) & ~15) + 96 + (((24 * nsmax) + 15) & ~15) + LB + TB + 16 + 512);
}

// The kernel unit: rx_pass1 (a CTA of 16 warps runs one group over 16
// consecutive segments), rx_prefilter, rx_fixup (phase 1: one warp per
// (group, segment); phase 2 and rematch: one warp per group).
std::string emit_kernel_unit(CompiledSet &cs, int gb, int ge) {
  std::ostringstream os;
  os << kDevicePrelude << "\n// ===================== kernels (groups " << gb << ".." << ge - 1
     << ") =====================\n";
  int G = (int)cs.groups.size();
  os << "#define RX_NG " << G << "\n#define RX_G0 " << gb << "\n#define RX_G1 " << ge << "\n";
  for (int gi = gb; gi < ge; ++gi) {
    os << "extern \"C\" __device__ void rx_seg_" << gi << "(int seg);\n";
    if (cs.groups[gi].nslots > 0) os << "extern \"C\" __device__ void rx_fix_" << gi << "(int seg);\n";
  }
  os << "\nextern \"C\" __global__ void __launch_bounds__(" << 32 * cs.pass1_warps << ", 1) rx_pass1(const RxParams p) {\n"
        "  const int warp = threadIdx.x >> 5;\n"
        "  const int wpb = blockDim.x >> 5;\n"
        "  const int cpg = (p.nseg_max + wpb - 1) / wpb;  // CTAs per group\n"
        "  const int g = RX_G0 + (int)(blockIdx.x / cpg);\n"
        "  const long long seg = (long long)(blockIdx.x % cpg) * wpb + warp;\n"
        "  if (g >= RX_G1) return;\n"
        "  rx_cta_params_store(p);\n"
        "  switch (g) {\n";
  for (int gi = gb; gi < ge; ++gi) os << "    case " << gi << ": rx_seg_" << gi << "((int)seg); break;\n";
  os << "    default: break;\n  }\n}\n";
  if (cs.use_pf)
    os << "\nextern \"C\" __global__ void __launch_bounds__(256, 3) rx_prefilter(const RxParams p) {\n"
          "  rx_prefilter_run(p, RX_NG);\n}\n";
  os << "\nextern \"C\" __global__ void __launch_bounds__(128) rx_fixup(const RxParams p) {\n"
        "  const int warp = threadIdx.x >> 5;\n"
        "  const int wpb = blockDim.x >> 5;\n"
        "  const long long gw = (long long)blockIdx.x * wpb + warp;\n"
        "  // phase 1: warp -> (group, segment); otherwise warp -> group\n"
        "  const long long g = RX_G0 + (p.fix_phase == 1 ? gw / p.nseg_max : gw);\n"
        "  const int seg = p.fix_phase == 1 ? (int)(gw % p.nseg_max) : 0;\n"
        "  rx_cta_params_store(p);\n"
        "  if (g >= RX_G1) return;\n"
        "  switch ((int)g) {\n";
  for (int gi = gb; gi < ge; ++gi)
    if (cs.groups[gi].nslots > 0) os << "    case " << gi << ": rx_fix_" << gi << "(seg); break;\n";
  os << "    default: break;\n  }\n}\n";
  return os.str();
}

}  // namespace rx
