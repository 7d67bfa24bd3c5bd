// rx_lower.cpp -- lowering regexes to the bitstream IR, margin analysis,
// Shift Rebalancing, zero-block guards, grouping.
//
// Lowering follows PAPER.md Fig. 2 in the end-position
// convention of P:L120 ("a 1 at position i indicates a successful match
// ending at that position"):
//   E(CC, M)        = Adv(M, 1) & CC                       Fig. 2b
//   E(R1|R2, M)     = E(R1, M) | E(R2, M)                  Fig. 2c
//   E(R{n,m}, M)    = unrolled concatenation, OR of the n..m chains  Fig. 2d
//   E(R+, M)        = while-fixpoint with frontier/acc     Fig. 2e, Listing 3
//   E(CC+, M)       = MatchStar (one add with carry)       Parabix [24]
// M = Ones is the unanchored start ("R1 is used as a prefix to determine the
// starting positions"; every position may start).  Only non-empty
// matches are produced (reading c1): R? and R* contribute their non-empty
// part; concatenation tracks P (prefix may be empty) and N (non-empty).
#include <algorithm>
#include <cassert>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <sstream>
#include <tuple>

#include "rx_internal.h"

namespace rx {
namespace {

struct Key {
  Op op;
  int a, b, k, cc;
  bool operator<(const Key &o) const {
    return std::tie(op, a, b, k, cc) < std::tie(o.op, o.a, o.b, o.k, o.cc);
  }
};

struct Item {
  const Ast *ast;
  enum Mode { Once, Opt, Plus } mode;
};

struct Lowerer {
  RegexIR &ir;
  LowerOptions opt;
  std::vector<int> blk;                     // block stack
  std::vector<int> loops;                   // enclosing loop nodes
  std::vector<std::map<Key, int>> cse;      // scoped hash-consing
  std::map<std::vector<uint64_t>, int> set_ix;
  std::map<std::string, int> lit_ix;
  int zero = -1, ones = -1;
  size_t since_guard = 0;

  Lowerer(RegexIR &r, const LowerOptions &o) : ir(r), opt(o) {}

  int cur_loop() const { return loops.empty() ? -1 : loops.back(); }

  int raw(Node n) {
    n.loop = cur_loop();
    ir.nodes.push_back(n);
    int id = (int)ir.nodes.size() - 1;
    ir.blocks[blk.back()].nodes.push_back(id);
    ir.n_instr++;
    since_guard++;
    return id;
  }

  int mk(Op op, int a = -1, int b = -1, int k = 0, int cc = -1) {
    if ((op == Op::And || op == Op::Or || op == Op::Xor) && a > b) std::swap(a, b);
    Key key{op, a, b, k, cc};
    for (auto it = cse.rbegin(); it != cse.rend(); ++it) {
      auto f = it->find(key);
      if (f != it->end()) return f->second;
    }
    Node n;
    n.op = op;
    n.a = a;
    n.b = b;
    n.k = k;
    n.cc = cc;
    int id = raw(n);
    cse.back()[key] = id;
    return id;
  }

  int push_block() {
    ir.blocks.emplace_back();
    int id = (int)ir.blocks.size() - 1;
    blk.push_back(id);
    cse.emplace_back();
    return id;
  }
  void pop_block() {
    blk.pop_back();
    cse.pop_back();
  }

  bool is(int v, Op op) const { return ir.nodes[v].op == op; }

  // --- constant-folding constructors -------------------------------------
  int Zero() { return zero; }
  int AND(int a, int b) {
    if (is(a, Op::Zero) || is(b, Op::Zero)) return zero;
    if (is(a, Op::Ones)) return b;
    if (is(b, Op::Ones)) return a;
    if (a == b) return a;
    return mk(Op::And, a, b);
  }
  int OR(int a, int b) {
    if (is(a, Op::Zero)) return b;
    if (is(b, Op::Zero)) return a;
    if (is(a, Op::Ones) || is(b, Op::Ones)) return ones;
    if (a == b) return a;
    return mk(Op::Or, a, b);
  }
  int ADV1(int m) {
    if (is(m, Op::Zero)) return zero;
    if (is(m, Op::Ones)) return ones;  // the virtual start at position -1 (P:L116 prefix)
    return mk(Op::Adv, m, -1, 1);
  }
  int CC(const ByteSet &s) {
    if (s.empty()) return zero;
    std::vector<uint64_t> key(s.w, s.w + 4);
    int ix;
    auto f = set_ix.find(key);
    if (f == set_ix.end()) {
      ix = (int)ir.sets.size();
      ir.sets.push_back(s);
      set_ix[key] = ix;
    } else {
      ix = f->second;
    }
    return mk(Op::CC, -1, -1, 0, ix);
  }

  int LIT(int m, const std::string &s) {
    if (is(m, Op::Zero)) return zero;
    int ix;
    auto f = lit_ix.find(s);
    if (f == lit_ix.end()) {
      ix = (int)ir.lits.size();
      ir.lits.push_back(s);
      lit_ix[s] = ix;
    } else {
      ix = f->second;
    }
    return mk(Op::Lit, m, -1, (int)s.size(), ix);
  }
  // a Once item matching exactly one byte value, not 0x00 (the Lit confirm
  // compares raw bytes; 0x00 is also the padding beyond the stream)
  static bool single_byte(const Item &it, int &c) {
    ByteSet s;
    if (it.mode != Item::Once || !single_set(*it.ast, s) || s.count() != 1) return false;
    for (int b = 1; b < 256; ++b)
      if (s.has(b)) {
        c = b;
        return true;
      }
    return false;
  }

  int ADVK(int m, int k) {
    if (k == 0) return m;
    if (is(m, Op::Zero)) return zero;
    if (is(m, Op::Ones)) return ones;
    return mk(Op::Adv, m, -1, k);
  }
  // Cr_t = positions q whose t bytes (q-t, q] are all in class C, by
  // doubling: Cr_{x+y} = Cr_x & Adv(Cr_y, x) (Fig. 2d's bounded repetition
  // unrolls this one byte at a time; the result is the same stream)
  int CRUN(int C, int t) {
    std::vector<int> pw = {C};  // pw[j] = Cr_{2^j}
    while ((1 << pw.size()) <= t) {
      int j = (int)pw.size() - 1;
      pw.push_back(AND(pw[j], ADVK(pw[j], 1 << j)));
    }
    int res = -1, len = 0;
    for (int j = (int)pw.size() - 1; j >= 0; --j)
      if ((t >> j) & 1) {
        res = res < 0 ? pw[j] : AND(res, ADVK(pw[j], len));
        len += 1 << j;
      }
    return res;
  }
  // E(C{lo,hi}, M), C a single class, hi >= 0: the non-empty ends q with
  // some p in M, max(lo,1) <= q-p <= hi and bytes (p, q] all in C.  Exact
  // distance a = max(lo,1) first (Y), then the reach S_t(Y) of up to t more
  // C bytes extended by doubling: S_{t+b} = S_t | (Adv(S_t, b) & Cr_b) for
  // b <= t+1.  O(log hi) operations instead of the (hi-lo) optional items of
  // Fig. 2d; the result is the same stream (tests: brute force over {n,m}).
  int E_crep(const ByteSet &cs, int lo, int hi, int M) {
    int C = CC(cs);
    int a = std::max(lo, 1);
    if (hi < a) return zero;
    int Y = is(M, Op::Ones) ? CRUN(C, a) : AND(ADVK(M, a), CRUN(C, a));
    int S = Y;
    for (int t = 0; t < hi - a && !is(S, Op::Zero);) {
      int b = std::min(t + 1, hi - a - t);
      S = OR(S, AND(ADVK(S, b), CRUN(C, b)));
      t += b;
    }
    return S;
  }

  // --- E(R, M) -------------------------------------------------------------
  static const Ast *single_set(const Ast &a, ByteSet &out) {
    // A sub-expression that matches exactly one byte from a set: Set, or
    // Alt of single sets, or Rep{1,1} of one.
    if (a.kind == AK::Set) { out = a.set; return &a; }
    if (a.kind == AK::Alt) {
      ByteSet u;
      for (auto &k : a.kids) {
        ByteSet s;
        if (!single_set(*k, s)) return nullptr;
        u.merge(s);
      }
      out = u;
      return &a;
    }
    if (a.kind == AK::Rep && a.lo == 1 && a.hi == 1) return single_set(*a.kids[0], out);
    if (a.kind == AK::Cat && a.kids.size() == 1) return single_set(*a.kids[0], out);
    return nullptr;
  }

  int E(const Ast &r, int M) {
    if (is(M, Op::Zero)) return zero;
    switch (r.kind) {
      case AK::Empty: return zero;
      case AK::Set: return AND(ADV1(M), CC(r.set));
      case AK::Alt: {
        int acc = zero;
        for (auto &k : r.kids) acc = OR(acc, E(*k, M));
        return acc;
      }
      case AK::Cat: {
        std::vector<Item> items;
        for (auto &k : r.kids) items.push_back({k.get(), Item::Once});
        return E_cat(items, 0, M, zero);
      }
      case AK::Rep: {
        const Ast &kid = *r.kids[0];
        if (r.hi == 0) return zero;
        {
          ByteSet cs;
          if (loops.empty() && single_set(kid, cs) && !cs.empty()) {
            if (r.hi >= 0 && (r.hi - std::max(r.lo, 1) >= 3 || r.lo >= 5)) return E_crep(cs, r.lo, r.hi, M);
            if (r.hi < 0 && r.lo >= 6) {
              // C{n,} = C{n-1} C+ : the fixed part by doubling, then MatchStar
              int C = CC(cs);
              int Y = is(M, Op::Ones) ? CRUN(C, r.lo - 1) : AND(ADVK(M, r.lo - 1), CRUN(C, r.lo - 1));
              return E_plus(kid, Y);
            }
          }
        }
        std::vector<Item> items;
        if (r.hi < 0) {
          for (int i = 0; i + 1 < r.lo; ++i) items.push_back({&kid, Item::Once});
          items.push_back({&kid, Item::Plus});
        } else {
          for (int i = 0; i < r.lo; ++i) items.push_back({&kid, Item::Once});
          for (int i = r.lo; i < r.hi; ++i) items.push_back({&kid, Item::Opt});
        }
        return E_cat(items, 0, M, zero);
      }
    }
    return zero;
  }

  int E_item(const Item &it, int P) {
    switch (it.mode) {
      case Item::Once:
      case Item::Opt: return E(*it.ast, P);
      case Item::Plus: return E_plus(*it.ast, P);
    }
    return zero;
  }
  bool item_nullable(const Item &it) {
    return it.mode == Item::Opt || ast_nullable(*it.ast);
  }

  // Concatenation items[j..] after a prefix whose (possibly empty) end
  // markers are P and whose non-empty end markers are N.
  int E_cat(const std::vector<Item> &items, size_t j, int P, int N, bool guarded = false, int single_run = 0) {
    // leading run of single-class items of an unanchored chain: unguarded
    // with opt.lead_noguard (LowerOptions)
    size_t lead = 0;
    if (opt.lead_noguard && j == 0 && is(P, Op::Ones) && loops.empty()) {
      ByteSet tmp;
      while (lead < items.size() && items[lead].mode == Item::Once && single_set(*items[lead].ast, tmp)) ++lead;
    }
    // single_run: single-byte items just consumed by this chain
    for (; j < items.size(); ++j) {
      // Zero-block-skipping guard (Sec. 6): P is a zero-path
      // head -- if P is all-zero in a window, everything downstream in this
      // concatenation (and N, a subset of P) is zero.  First guard at the
      // head of the path (after its first shift+AND), then every `interval`
      // instructions.
      const bool head = !guarded && ir.nodes[P].op == Op::And;
      if (opt.interval > 0 && loops.empty() && j > 0 && j >= lead && !is(P, Op::Ones) && !is(P, Op::Zero) &&
          (head || since_guard >= (size_t)opt.interval) && ir.nodes[P].op != Op::CC) {
        Node g;
        g.op = Op::Guard;
        g.a = P;
        int gid = raw(g);
        ir.n_guards++;
        int sb = push_block();
        since_guard = 0;
        int res = E_cat(items, j, P, N, true, single_run);
        pop_block();
        ir.nodes[gid].sub = sb;
        ir.nodes[gid].res = res;
        if (is(res, Op::Zero)) return zero;
        return gid;
      }
      // literal run (LowerOptions::lit_after / lit_min): one Lit node
      int cb = 0;
      if (opt.lit_min > 0 && loops.empty() && single_run >= opt.lit_after && !is(P, Op::Ones) &&
          single_byte(items[j], cb)) {
        std::string s;
        size_t r = j;
        for (int c2 = 0; r < items.size() && single_byte(items[r], c2); ++r) s += (char)c2;
        if ((int)s.size() >= opt.lit_min) {
          P = N = LIT(P, s);
          single_run += (int)s.size();
          j = r - 1;
          if (is(P, Op::Zero)) return zero;
          continue;
        }
      }
      const Item &it = items[j];
      {
        int c3 = 0;
        single_run = single_byte(it, c3) ? single_run + 1 : 0;
      }
      int e = E_item(it, P);
      if (item_nullable(it)) {
        int nP = OR(e, P);
        N = OR(e, N);
        P = nP;
      } else {
        P = e;
        N = e;
      }
      if (is(P, Op::Zero)) return zero;
    }
    return N;
  }

  // E(R+, M): non-empty repetitions of R after prefix ends M.
  int E_plus(const Ast &r, int M) {
    ByteSet s;
    if (single_set(r, s)) {
      if (s.empty()) return zero;
      int C = CC(s);
      if (is(M, Op::Ones)) return C;  // every C position ends a one-byte match
      int X = AND(ADV1(M), C);
      if (is(X, Op::Zero)) return zero;
      Node n;
      n.op = Op::MStar;
      n.a = X;
      n.b = C;
      ir.n_mstar++;
      return raw(n);  // stateful: never hash-consed
    }
    // General body: while-fixpoint (Fig. 2e, Listing 3).  The frontier
    // starts at the prefix ends M itself, so the body E(r, .) is lowered
    // once: acc = U_i E(r, fr_i), fr_0 = M, fr_{i+1} = E(r, fr_i) & ~acc.
    // (At the unanchored start M = Ones, seed the loop with E(r, Ones) --
    // the virtual start position has no bit in the window.)
    int seeds = M;
    if (is(M, Op::Ones)) {
      int e = E(r, M);
      if (is(e, Op::Zero)) return zero;
      Node L0;
      L0.op = Op::Loop;
      L0.a = e;
      L0.k = 1;  // k=1: seeds are ends of r already (acc starts with them)
      int lid0 = raw(L0);
      ir.n_loops++;
      lower_body(lid0, r);
      return lid0;
    }
    Node L;
    L.op = Op::Loop;
    L.a = seeds;
    L.k = 0;  // k=0: seeds are prefix ends (frontier only, not in acc)
    int lid = raw(L);
    ir.n_loops++;
    lower_body(lid, r);
    return lid;
  }

  void lower_body(int lid, const Ast &r) {
    int sb = push_block();
    loops.push_back(lid);
    Node f;
    f.op = Op::Fr;
    int fr = raw(f);
    int res = E(r, fr);
    loops.pop_back();
    pop_block();
    ir.nodes[lid].sub = sb;
    ir.nodes[lid].fr = fr;
    ir.nodes[lid].res = res;
  }
};

}  // namespace

void lower_cluster(const std::vector<const Ast *> &asts, const LowerOptions &opt, RegexIR &ir) {
  ir = RegexIR();
  ir.blocks.emplace_back();
  Lowerer L(ir, opt);
  L.blk.push_back(0);
  L.cse.emplace_back();
  Node z;
  z.op = Op::Zero;
  L.zero = L.raw(z);
  Node o;
  o.op = Op::Ones;
  L.ones = L.raw(o);
  ir.n_instr = 0;
  for (const Ast *a : asts) {
    L.since_guard = 0;
    int out = L.E(*a, L.ones);
    if (out == L.ones) {
      // a regex matching every position with a one-byte match of [\x00-\xff]
      // cannot lower to Ones (Ones is 1 at padding too); E never returns Ones
      // for a non-empty R, keep the guard anyway.
      out = L.CC([] { ByteSet s; s.range(0, 255); return s; }());
    }
    ir.outs.push_back(out);
  }
  ir.out = ir.outs.empty() ? L.zero : ir.outs[0];
}

void lower_regex(const Ast &ast, const LowerOptions &opt, RegexIR &ir) { lower_cluster({&ast}, opt, ir); }

// ----------------------------------------------------------------------------
// Margins: a window frame computes words [0, 32K); a
// value v is exact at bit positions [lb(v), 32K*32 - rb(v)).  Static shifts
// grow the margins (the paper's overlap distance, generalised to
// per-side margins, SURVEY App.A-8); unbounded constructs (MatchStar, while
// loops) are exact from their injection word aw on, with their cross-window
// dependency carried as state.
// ----------------------------------------------------------------------------
static void mark_loop_sites(RegexIR &ir, int block, int aw, int &slot) {
  for (int id : ir.blocks[block].nodes) {
    Node &n = ir.nodes[id];
    switch (n.op) {
      case Op::Adv:
        if (n.k > 32) n.k = 32;  // (bodies only produce Adv 1)
        n.aw = aw;
        n.slot = slot++;
        break;
      case Op::MStar:
        n.aw = aw;
        n.slot = slot++;
        break;
      case Op::Loop:
        n.aw = aw;
        mark_loop_sites(ir, n.sub, aw, slot);
        break;
      case Op::Guard:
        mark_loop_sites(ir, n.sub, aw, slot);
        break;
      default:
        break;
    }
  }
}

static void margins_block(RegexIR &ir, int block, int &slot) {
  for (int id : ir.blocks[block].nodes) {
    Node &n = ir.nodes[id];
    auto lb = [&](int x) { return ir.nodes[x].lb; };
    auto rb = [&](int x) { return ir.nodes[x].rb; };
    auto dp = [&](int x) { return ir.nodes[x].depth; };
    switch (n.op) {
      case Op::Zero: case Op::Ones: case Op::CC: case Op::Fr:
        n.lb = n.rb = 0;
        n.depth = 0;
        break;
      case Op::And: case Op::Or: case Op::Xor: case Op::AndNot:
        n.lb = std::max(lb(n.a), lb(n.b));
        n.rb = std::max(rb(n.a), rb(n.b));
        n.depth = std::max(dp(n.a), dp(n.b)) + 1;
        break;
      case Op::Adv:
        n.lb = lb(n.a) + n.k;
        n.rb = std::max(rb(n.a) - n.k, 0);
        n.depth = dp(n.a) + 1;
        break;
      case Op::Lit:  // = k advances by one (and ANDs with classes)
        n.lb = lb(n.a) + n.k;
        n.rb = std::max(rb(n.a) - n.k, 0);
        n.depth = dp(n.a) + 1;
        break;
      case Op::Look:
        n.lb = std::max(lb(n.a) - n.k, 0);
        n.rb = rb(n.a) + n.k;
        n.depth = dp(n.a) + 1;
        break;
      case Op::MStar: {
        int l = std::max(lb(n.a), lb(n.b));
        n.aw = (l + 31) / 32;
        n.slot = slot++;
        n.lb = 32 * n.aw;
        n.rb = std::max(rb(n.a), rb(n.b));
        n.depth = std::max(dp(n.a), dp(n.b)) + 4;
        ir.rb_state = std::max(ir.rb_state, n.rb);
        break;
      }
      case Op::Loop: {
        // body invariants are CCs (lb 0); seeds carry the static part
        n.aw = (lb(n.a) + 31) / 32 + 1;
        mark_loop_sites(ir, n.sub, n.aw, slot);
        n.lb = 32 * n.aw;
        n.rb = rb(n.a);
        n.depth = dp(n.a) + 8;
        ir.rb_state = std::max(ir.rb_state, n.rb);
        break;
      }
      case Op::Guard: {
        margins_block(ir, n.sub, slot);
        n.lb = lb(n.res);
        n.rb = rb(n.res);
        n.depth = dp(n.res);
        break;
      }
    }
  }
}

bool analyze_regex(RegexIR &ir, std::string &why) {
  int slot = 0;
  margins_block(ir, 0, slot);
  ir.nslots = slot;
  ir.lb = ir.rb = 0;
  for (int o : ir.outs) {
    ir.lb = std::max(ir.lb, ir.nodes[o].lb);
    ir.rb = std::max(ir.rb, ir.nodes[o].rb);
  }
  (void)why;
  return true;
}

std::string dump_ir(const RegexIR &ir) {
  static const char *names[] = {"zero", "ones", "cc", "and", "or", "xor", "andn", "adv", "look",
                                "mstar", "loop", "fr", "guard", "lit"};
  std::ostringstream os;
  std::function<void(int, int)> blk = [&](int b, int ind) {
    for (int id : ir.blocks[b].nodes) {
      const Node &n = ir.nodes[id];
      os << std::string(ind, ' ') << "v" << id << " = " << names[(int)n.op];
      if (n.a >= 0) os << " v" << n.a;
      if (n.b >= 0) os << " v" << n.b;
      if (n.op == Op::Adv || n.op == Op::Look) os << " k=" << n.k;
      if (n.op == Op::CC) os << " set#" << n.cc;
      if (n.op == Op::Lit) os << " k=" << n.k << " lit#" << n.cc;
      os << "   [lb=" << n.lb << " rb=" << n.rb;
      if (n.slot >= 0) os << " slot=" << n.slot << " aw=" << n.aw;
      if (n.loop >= 0) os << " in-loop v" << n.loop;
      os << "]\n";
      if (n.op == Op::Loop || n.op == Op::Guard) {
        blk(n.sub, ind + 2);
        os << std::string(ind + 2, ' ') << "-> v" << n.res << "\n";
      }
    }
  };
  blk(0, 0);
  os << "out = v" << ir.out << " lb=" << ir.lb << " rb=" << ir.rb << " slots=" << ir.nslots << "\n";
  return os.str();
}

// ----------------------------------------------------------------------------
// Grouping ("Regexes are partitioned into groups with similar
// total character length, each assigned to one CTA").  Here a group is the
// program one warp runs over its windows; regexes are sorted by static span
// so that a group's window geometry (K, halos) fits all members, then packed
// greedily by instruction count.
// ----------------------------------------------------------------------------
bool plan_groups(CompiledSet &cs, int group_size, int force_K, std::string &why) {
  int n = (int)cs.irs.size();
  std::vector<int> order(n);
  for (int i = 0; i < n; ++i) order[i] = i;
  auto span = [&](int r) { return (cs.irs[r].lb + 31) / 32 + (std::max(cs.irs[r].rb, cs.irs[r].rb_state) + 31) / 32; };
  // window-width class first (a group's geometry must fit every member),
  // then -- with the prefilter -- members without a factor apart from the
  // others (their groups run every window), and members sharing a factor
  // together (one factor hit then wakes one group)
  auto kclass = [&](int r) {
    const int w = span(r);
    for (int k : {2, 4, 8})
      if (4 * w <= 32 * k) return k;
    return 16;
  };
  auto fac = [&](int r) { return cs.factor_of.empty() ? -1 : cs.factor_of[r]; };
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) {
    if (kclass(a) != kclass(b)) return kclass(a) < kclass(b);
    if ((fac(a) < 0) != (fac(b) < 0)) return fac(a) < 0;
    if (fac(a) != fac(b)) return fac(a) < fac(b);
    return span(a) < span(b);
  });
  size_t total_instr = 0;
  for (auto &r : cs.irs) total_instr += r.n_instr;
  if (group_size <= 0 || group_size > 32) group_size = 32;  // member masks are 32-bit
  // bounds one NVRTC unit (compile time) and the group's code size (the
  // SM's instruction caches hold one group's program; measured flat over
  // 600-3000)
  const size_t max_instr = 1500;
  cs.groups.clear();
  Group g;
  size_t gi = 0;
  for (int r : order) {
    const bool split_always = !g.regexes.empty() && (fac(g.regexes.back()) < 0) != (fac(r) < 0);
    if (!g.regexes.empty() &&
        ((int)g.regexes.size() >= group_size || gi + cs.irs[r].n_instr > max_instr || split_always)) {
      cs.groups.push_back(g);
      g = Group();
      gi = 0;
    }
    g.regexes.push_back(r);
    gi += cs.irs[r].n_instr;
    g.cost += (double)cs.irs[r].n_instr;
  }
  if (!g.regexes.empty() || cs.groups.empty()) cs.groups.push_back(g);
  for (auto &gr : cs.groups) {
    int L = 0, R = 0;
    gr.nslots = 0;
    gr.slot_base.clear();
    gr.always = 0;
    gr.out_delta = 0;
    for (int r : gr.regexes) {
      const RegexIR &ir = cs.irs[r];
      if (fac(r) < 0) gr.always |= 1u << gr.slot_base.size();
      L = std::max(L, (ir.lb + 31) / 32);
      // mode B (output-gated) needs every output-factor anchor of a match
      // ending in the committed range inside the frame: Lw words >= delta
      if (!cs.rf.empty() && !cs.rf[r].out.empty()) {
        gr.out_delta = std::max(gr.out_delta, cs.rf[r].out_delta);
        L = std::max(L, (cs.rf[r].out_delta + 31) / 32);
      }
      R = std::max(R, (std::max(ir.rb, ir.rb_state) + 31) / 32);
      gr.slot_base.push_back(gr.nslots);
      gr.nslots += ir.nslots;
    }
    // K (words per lane): the smallest power of two >= the requested minimum
    // (default 2: two independent words per lane per instruction, per-window
    // costs amortised over 2048 positions) whose halo overhead is <= 25%
    const int min_K = force_K > 0 ? force_K : 2;
    int K = 8;
    for (int k : {1, 2, 4, 8})
      if (k >= min_K && 4 * (L + R) <= 32 * k) { K = k; break; }
    if (K < min_K) K = min_K;
    if (L + R >= 32 * K) {
      why = "static span of a group exceeds the window (" + std::to_string(L + R) + " words)";
      return false;
    }
    gr.K = K;
    gr.Lw = L;
    gr.Rw = R;
    gr.Bw = 32 * K - L - R;
  }
  return true;
}

// Factor clusters: inside a group, members with the
// same prefilter factor are woken by the same hits, so they are lowered
// together and their common prefix (shared CCs, shifts and ANDs up to the
// first zero-block guard) is computed once per window; members without a
// factor form one cluster that runs in every window.
bool build_clusters(CompiledSet &cs, const std::vector<const Ast *> &asts, const LowerOptions &opt,
                    std::string &why) {
  for (auto &g : cs.groups) {
    g.clusters.clear();
    // cluster key: (first-factor set, has output factors) -- a cluster runs
    // output-gated (mode B) only if all of its members can
    std::map<std::pair<int, bool>, int> by_factor;
    for (size_t m = 0; m < g.regexes.size(); ++m) {
      const int r = g.regexes[m];
      const int f = cs.factor_of.empty() ? -1 : cs.factor_of[r];
      const bool bc = !cs.rf.empty() && !cs.rf[r].out.empty();
      auto it = by_factor.find({f, bc});
      int ci;
      if (it == by_factor.end()) {
        ci = (int)g.clusters.size();
        by_factor[{f, bc}] = ci;
        g.clusters.emplace_back();
        g.clusters.back().always = f < 0;
        g.clusters.back().bcap = bc;
      } else {
        ci = it->second;
      }
      g.clusters[ci].members.push_back((int)m);
    }
    int L = 0, R = 0;
    g.nslots = 0;
    for (auto &c : g.clusters) {
      std::vector<const Ast *> as;
      for (int m : c.members) as.push_back(asts[g.regexes[m]]);
      LowerOptions co = opt;
      co.lead_noguard = opt.lead_noguard && !c.always;
      lower_cluster(as, co, c.ir);
      if (opt.rebalance) rebalance_regex(c.ir);
      if (!analyze_regex(c.ir, why)) return false;
      c.slot_base = g.nslots;
      g.nslots += c.ir.nslots;
      L = std::max(L, (c.ir.lb + 31) / 32);
      R = std::max(R, (std::max(c.ir.rb, c.ir.rb_state) + 31) / 32);
    }
    if (L > g.Lw || R > g.Rw) {
      why = "cluster margins exceed the group window";
      return false;
    }
  }
  return true;
}

}  // namespace rx
