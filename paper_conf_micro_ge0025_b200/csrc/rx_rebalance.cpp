// rx_rebalance.cpp -- Shift Rebalancing (Sec. 5.2).
//
// Operand rewriting: (A >> n) & B  ==  (A & (B << n)) >> n, exact on
// finite zero-padded streams (SURVEY App.A-5).  The pass traverses the DFG in
// topological order; for every AND whose operand is an Advance deeper than
// the other operand B (depth(A) + 1 > depth(B)), the Advance is moved onto B
// as a lookahead and applied after the AND ("the SHIFT ... is moved to the
// operand with lower topological depth"), iterating to a fixpoint;
// trailing Advances of Advances are merged afterwards ("merged after
// the last AND").
//
// Only top-level / guard-region code is rewritten: inside while-loop bodies
// every Advance is a forwarded cross-window site and a
// lookahead would need future windows.  On B200 the payoff is instruction-
// level parallelism (shorter dependence chains of shuffles), not barrier count
// -- at warp scope shifts need no barriers.
#include <algorithm>
#include <vector>

#include "rx_internal.h"

namespace rx {
namespace {

struct Pass {
  RegexIR &ir;
  std::vector<int> depth;
  explicit Pass(RegexIR &r) : ir(r) {}

  int d(int x) const { return x < 0 ? 0 : depth[x]; }

  void compute_depth(int block) {
    for (int id : ir.blocks[block].nodes) {
      const Node &n = ir.nodes[id];
      int v = 0;
      switch (n.op) {
        case Op::Zero: case Op::Ones: case Op::CC: case Op::Fr: v = 0; break;
        case Op::Guard: compute_depth(n.sub); v = d(n.res); break;
        case Op::Loop: compute_depth(n.sub); v = d(n.a) + 1; break;
        default: v = std::max(d(n.a), d(n.b)) + 1; break;
      }
      depth[id] = v;
    }
  }

  int add(int block, size_t pos, Node n) {
    n.loop = -1;
    ir.nodes.push_back(n);
    depth.push_back(0);
    int id = (int)ir.nodes.size() - 1;
    auto &v = ir.blocks[block].nodes;
    v.insert(v.begin() + (long)pos, id);
    return id;
  }

  // one sweep over a block (and nested guard regions); returns #rewrites
  int sweep(int block) {
    int changed = 0;
    for (size_t i = 0; i < ir.blocks[block].nodes.size(); ++i) {
      int id = ir.blocks[block].nodes[i];
      Node &n = ir.nodes[id];
      if (n.op == Op::Guard) {
        changed += sweep(n.sub);
        continue;
      }
      if (n.op != Op::And || n.loop >= 0) continue;
      for (int side = 0; side < 2; ++side) {
        int x = side ? n.b : n.a, y = side ? n.a : n.b;
        const Node &nx = ir.nodes[x];
        if (nx.op != Op::Adv || nx.loop >= 0 || nx.k <= 0) continue;
        int A = nx.a, k = nx.k;
        // the SHIFT operand (depth d(A) + 1) is deeper than the other one
        if (!(d(A) + 1 > d(y))) continue;
        Node look;
        look.op = Op::Look;
        look.a = y;
        look.k = k;
        int L = add(block, i, look);
        Node t;
        t.op = Op::And;
        t.a = A;
        t.b = L;
        int T = add(block, i + 1, t);
        Node &m = ir.nodes[id];  // (re-fetch: the vector may have grown)
        m.op = Op::Adv;
        m.a = T;
        m.b = -1;
        m.k = k;
        depth[L] = d(y) + 1;
        depth[T] = std::max(d(A), depth[L]) + 1;
        depth[id] = depth[T] + 1;
        i += 2;
        ++changed;
        break;
      }
    }
    return changed;
  }

  // Adv(Adv(x, a), b) -> Adv(x, a + b) when the inner Advance is top-level
  void merge(int block) {
    for (int id : ir.blocks[block].nodes) {
      Node &n = ir.nodes[id];
      if (n.op == Op::Guard) {
        merge(n.sub);
        continue;
      }
      if ((n.op == Op::Adv || n.op == Op::Look) && n.loop < 0) {
        const Node &in = ir.nodes[n.a];
        if (in.op == n.op && in.loop < 0 && n.k + in.k <= 1024) {
          n.k += in.k;
          n.a = in.a;
        }
      }
    }
  }
};

}  // namespace

void rebalance_regex(RegexIR &ir) {
  Pass p(ir);
  for (int it = 0; it < 16; ++it) {
    p.depth.assign(ir.nodes.size(), 0);
    p.compute_depth(0);
    if (p.sweep(0) == 0) break;
  }
  p.merge(0);
}

}  // namespace rx
