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

// Device tables of the prefilter, one u32 blob (layout documented at
// RxParams::pf_tab in rx_device.cuh):
//   l1[2048]     bitmap over the 65,536 bigrams: each gram's index bigram
//                (its rarest byte pair under the model)
//   rank[2048]   set bits of l1 before word i (compact index of a set bigram)
//   bsid[nb]     per set bigram: mask of the gram shapes indexed by it; shape
//                s = 3*(k-2) + d (k = gram length, d = gram bytes after the
//                index bigram)
//   htab[2*HS]   open-addressing hash set of (gram, shape) -> factor:
//                {gram, factor << 8 | shape << 1 | 1}; empty slots are 0
//   fgoff[nf+1]  per factor: its range of (group, member mask) pairs
//   fgent[2*m]
uint32_t pf_hash(uint32_t gram, uint32_t shape) { return (gram ^ (shape * 0x85EBCA6Bu)) * 0x9E3779B1u; }

void build_prefilter(CompiledSet &cs) {
  Prefilter &pf = cs.pf;
  pf = Prefilter();
  const int nf = (int)cs.factors.size();
  pf.nfactor = nf;
  std::vector<uint32_t> l1(2048, 0u);
  std::map<uint32_t, uint32_t> sids;  // index bigram -> shape mask
  struct E { uint32_t gram, shape, fid; };
  std::vector<E> ents;
  const Model &mdl = model();
  for (int f = 0; f < nf; ++f)
    for (auto &g : cs.factors[f].grams) {
      int best_d = 0;
      double best_p = 2.0;
      for (int d = 0; d + 2 <= g.k; ++d) {
        const int b1 = (g.gram >> (8 * (2 - d))) & 255, b2 = (g.gram >> (8 * (3 - d))) & 255;
        const double pp = mdl.p[b1] * mdl.p[b2];
        if (pp < best_p) {
          best_p = pp;
          best_d = d;
        }
      }
      const uint32_t bg = (g.gram >> (8 * (2 - best_d))) & 0xffffu;
      const uint32_t shape = 3u * (uint32_t)(g.k - 2) + (uint32_t)best_d;
      l1[bg >> 5] |= 1u << (bg & 31);
      sids[bg] |= 1u << shape;
      ents.push_back(E{g.gram, shape, (uint32_t)f});
    }
  std::vector<uint32_t> &B = pf.blob;
  B = l1;
  uint32_t run = 0;
  for (int i = 0; i < 2048; ++i) {
    B.push_back(run);
    run += (uint32_t)__builtin_popcount(l1[i]);
  }
  for (auto &kv : sids) B.push_back(kv.second);  // ascending bigram = ascending rank
  uint32_t hs = 64;
  while (hs < 2 * ents.size()) hs <<= 1;
  pf.hbits = 0;
  while ((1u << pf.hbits) < hs) ++pf.hbits;
  pf.o_ent = (uint32_t)B.size();
  std::vector<uint32_t> ht(2 * hs, 0u);
  for (auto &e : ents) {
    uint32_t h = pf_hash(e.gram, e.shape) >> (32 - pf.hbits);
    while (ht[2 * h + 1] != 0u) h = (h + 1) & (hs - 1);
    ht[2 * h] = e.gram;
    ht[2 * h + 1] = (e.fid << 8) | (e.shape << 1) | 1u;
  }
  B.insert(B.end(), ht.begin(), ht.end());
  // factor -> groups
  std::vector<std::map<int, uint32_t>> fg(nf);
  for (int gi = 0; gi < (int)cs.groups.size(); ++gi) {
    const Group &g = cs.groups[gi];
    for (size_t m = 0; m < g.regexes.size(); ++m) {
      const int f = cs.factor_of[g.regexes[m]];
      if (f >= 0) fg[f][gi] |= 1u << m;
    }
  }
  pf.o_fgoff = (uint32_t)B.size();
  std::vector<uint32_t> fge;
  for (int f = 0; f < nf; ++f) {
    B.push_back((uint32_t)(fge.size() / 2));
    for (auto &kv : fg[f]) fge.insert(fge.end(), {(uint32_t)kv.first, kv.second});
  }
  B.push_back((uint32_t)(fge.size() / 2));
  pf.o_fgent = (uint32_t)B.size();
  B.insert(B.end(), fge.begin(), fge.end());
}

}  // namespace rx
