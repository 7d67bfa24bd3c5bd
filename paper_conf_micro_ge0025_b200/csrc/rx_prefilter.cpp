// rx_prefilter.cpp -- the cross-regex literal prefilter (SURVEY.md Sec. 8(f)
// row N1, "hierarchical zero skipping"): host-side factor analysis and the
// device tables.
//
// Why: the interleaved kernel is integer-ALU bound ("the
// speedup tracks TIOPS"); Zero Block Skipping (Sec. 6) still pays
// each regex's guard head in every block, so the executed work grows with the
// number of regexes.  The paper names regex-specific work reduction such as
// literal matching as orthogonal and compatible.  Here one
// streaming pass over the input (rx_prefilter, rx_device.cuh) finds, for
// every 1 KiB block, which regex *factors* occur in it; the interleaved pass
// then runs a group in a window only if a member's factor occurs in the
// window's frame or a member carries state into it, and inside the window
// only those members.
//
// Soundness: a factor of regex r is a set of literal
// k-grams (2 <= k <= 4) such that
//   (i)  every string of L(r) contains one of them, and
//   (ii) every partial match that reaches a state slot (MatchStar carry,
//        while-loop frontier) contains one of them,
// taken from the mandatory single-byte-class runs of r's top-level
// concatenation *before its first unbounded repetition* (no state slot
// precedes that point, so any cursor held in a slot has consumed the run).
// With zero incoming state every 1-bit of a window's committed output or of
// its outgoing state is produced from class bits inside the window frame
// (margins keep halo garbage out of valid bits), i.e. from an actual (partial)
// match lying inside the frame -- which then contains a factor occurrence
// inside the frame.  So "no factor in the frame and no state in" implies
// "zero output and zero state out": skipping is exact.
#include <algorithm>
#include <cmath>
#include <map>

#include "rx_internal.h"

namespace rx {
namespace {

// A fixed model of byte frequencies in network payload / text, used only to
// rank candidate factors (rarer first).  Not data-dependent.
double byte_weight(int b) {
  if (b >= 'a' && b <= 'z') return 3.0;
  if (b == ' ') return 4.0;
  if (b >= 'A' && b <= 'Z') return 1.2;
  if (b >= '0' && b <= '9') return 1.5;
  if (b == '\n' || b == '\r' || b == '\t') return 1.0;
  if (b == '.' || b == '/' || b == '-' || b == ':' || b == '=' || b == '&' || b == '?' || b == '%' || b == '_' ||
      b == ',' || b == ';' || b == '+')
    return 1.0;
  if (b >= 0x20 && b < 0x7f) return 0.5;
  return 0.15;
}

struct Model {
  double p[256];
  Model() {
    double s = 0;
    for (int b = 0; b < 256; ++b) s += byte_weight(b);
    for (int b = 0; b < 256; ++b) p[b] = byte_weight(b) / s;
  }
  double set_p(const ByteSet &s) const {
    double v = 0;
    for (int b = 0; b < 256; ++b)
      if (s.has(b)) v += p[b];
    return v;
  }
};
const Model &model() {
  static Model m;
  return m;
}

bool has_unbounded(const Ast &a) {
  if (a.kind == AK::Rep && a.hi < 0) return true;
  for (auto &k : a.kids)
    if (has_unbounded(*k)) return true;
  return false;
}

bool single_set(const Ast &a, ByteSet &out) {
  if (a.kind == AK::Set) { out = a.set; return true; }
  if (a.kind == AK::Alt) {
    ByteSet u;
    for (auto &k : a.kids) {
      ByteSet s;
      if (!single_set(*k, s)) return false;
      u.merge(s);
    }
    out = u;
    return !a.kids.empty();
  }
  if (a.kind == AK::Rep && a.lo == 1 && a.hi == 1) return single_set(*a.kids[0], out);
  if (a.kind == AK::Cat && a.kids.size() == 1) return single_set(*a.kids[0], out);
  return false;
}

// Mandatory runs of byte classes along a concatenation, up to the first
// unbounded repetition.  `stop` is set once that point is reached.
struct RunCollector {
  std::vector<std::vector<ByteSet>> runs;
  std::vector<ByteSet> cur;
  bool stop = false;
  void brk() {
    if (!cur.empty()) runs.push_back(cur);
    cur.clear();
  }
  void item(const Ast &a) {
    if (stop) return;
    ByteSet s;
    if (single_set(a, s)) {
      cur.push_back(s);
      return;
    }
    switch (a.kind) {
      case AK::Empty: return;
      case AK::Cat:
        for (auto &k : a.kids) {
          item(*k);
          if (stop) return;
        }
        return;
      case AK::Rep:
        if (has_unbounded(a)) {  // the first state-carrying construct: the prefix ends here
          brk();
          stop = true;
          return;
        }
        for (int i = 0; i < a.lo && i < 8 && !stop; ++i) item(*a.kids[0]);
        if (a.hi != a.lo || a.lo > 8) brk();
        return;
      case AK::Alt:
      default:
        brk();
        if (has_unbounded(a)) stop = true;
        return;
    }
  }
};

struct Cand {
  std::vector<FactorGram> grams;
  double score = 1e30;
};

// best k-gram window of the runs (rarest under the model)
bool best_in_runs(const std::vector<std::vector<ByteSet>> &runs, Cand &best) {
  const Model &m = model();
  bool found = false;
  for (auto &run : runs) {
    for (int k = 4; k >= 2; --k) {
      const size_t cap = k == 2 ? 256 : 64;
      for (size_t i = 0; i + k <= run.size(); ++i) {
        size_t prod = 1;
        double sc = 1.0;
        for (int j = 0; j < k; ++j) {
          prod *= (size_t)run[i + j].count();
          sc *= m.set_p(run[i + j]);
          if (prod > cap) break;
        }
        if (prod > cap || prod == 0) continue;
        if (found && sc >= best.score) continue;
        // enumerate the k-grams: byte j of the gram at bit 8*(4-k+j) (the
        // gram ends at the last byte of the device's 4-byte window)
        std::vector<FactorGram> g(1, FactorGram{0u, 0u, k});
        for (int j = 0; j < k; ++j) {
          std::vector<FactorGram> ng;
          for (int b = 0; b < 256; ++b)
            if (run[i + j].has(b))
              for (auto &x : g) ng.push_back(FactorGram{x.gram | ((uint32_t)b << (8 * (4 - k + j))), 0u, k});
          g.swap(ng);
        }
        const uint32_t mask = k == 4 ? 0xffffffffu : (0xffffffffu << (8 * (4 - k)));
        for (auto &x : g) x.mask = mask;
        best.grams = g;
        best.score = sc;
        found = true;
      }
    }
  }
  return found;
}

bool factor_of(const Ast &a, Cand &out) {
  // top-level alternation: one factor per alternative, united
  if (a.kind == AK::Alt) {
    ByteSet s;
    if (!single_set(a, s)) {
      Cand u;
      u.score = 0;
      for (auto &k : a.kids) {
        Cand c;
        if (!factor_of(*k, c)) return false;
        u.grams.insert(u.grams.end(), c.grams.begin(), c.grams.end());
        u.score += c.score;
      }
      out = u;
      return !u.grams.empty();
    }
  }
  RunCollector rc;
  rc.item(a);
  rc.brk();
  return best_in_runs(rc.runs, out);
}

}  // namespace

bool regex_factor(const Ast &a, Factor &f) {
  Cand c;
  if (!factor_of(a, c)) return false;
  // a factor this common flags nearly every window: the regex always runs
  if (c.score > 0.02 || c.grams.size() > 512) return false;
  std::sort(c.grams.begin(), c.grams.end(), [](const FactorGram &x, const FactorGram &y) {
    return x.mask != y.mask ? x.mask < y.mask : x.gram < y.gram;
  });
  c.grams.erase(std::unique(c.grams.begin(), c.grams.end(),
                            [](const FactorGram &x, const FactorGram &y) {
                              return x.mask == y.mask && x.gram == y.gram;
                            }),
                c.grams.end());
  f.grams = c.grams;
  f.score = c.score;
  return true;
}

// Device tables of the prefilter (layout documented in rx_device.cuh,
// rx_prefilter kernel):
//   l1[2048]        bitmap over the 65,536 bigrams = last two bytes of a gram
//   e_off[65537]    CSR over that bigram -> entries
//   ent[4*n]        {gram, mask, factor id, k}
//   fg_off[nf+1]    CSR over factors -> (group, member mask) pairs
//   fg_ent[2*m]
void build_prefilter(CompiledSet &cs) {
  Prefilter &pf = cs.pf;
  pf = Prefilter();
  const int nf = (int)cs.factors.size();
  pf.nfactor = nf;
  pf.l1.assign(2048, 0u);
  std::vector<std::vector<uint32_t>> by_bg(65536);
  for (int f = 0; f < nf; ++f)
    for (auto &g : cs.factors[f].grams) {
      const uint32_t bg = g.gram >> 16;
      pf.l1[bg >> 5] |= 1u << (bg & 31);
      by_bg[bg].insert(by_bg[bg].end(), {g.gram, g.mask, (uint32_t)f, (uint32_t)g.k});
    }
  pf.e_off.assign(65537, 0u);
  for (int b = 0; b < 65536; ++b) {
    pf.e_off[b] = (uint32_t)(pf.ent.size() / 4);
    pf.ent.insert(pf.ent.end(), by_bg[b].begin(), by_bg[b].end());
  }
  pf.e_off[65536] = (uint32_t)(pf.ent.size() / 4);
  // factor -> groups
  std::vector<std::map<int, uint32_t>> fg(nf);
  for (int gi = 0; gi < (int)cs.groups.size(); ++gi) {
    const Group &g = cs.groups[gi];
    for (size_t m = 0; m < g.regexes.size(); ++m) {
      const int f = cs.factor_of[g.regexes[m]];
      if (f >= 0) fg[f][gi] |= 1u << m;
    }
  }
  pf.fg_off.assign(nf + 1, 0u);
  for (int f = 0; f < nf; ++f) {
    pf.fg_off[f] = (uint32_t)(pf.fg_ent.size() / 2);
    for (auto &kv : fg[f]) pf.fg_ent.insert(pf.fg_ent.end(), {(uint32_t)kv.first, kv.second});
  }
  pf.fg_off[nf] = (uint32_t)(pf.fg_ent.size() / 2);
}

}  // namespace rx
