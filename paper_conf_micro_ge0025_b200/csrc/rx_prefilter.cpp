// rx_prefilter.cpp -- the cross-regex literal prefilter (SURVEY.md Sec. 8(f)
// row N1, "hierarchical zero skipping"): host-side factor analysis and the
// device tables.
//
// Why: the interleaved kernel's work grows with the number of regexes; Zero
// Block Skipping (Sec. 6) still pays each regex's guard head in
// every block.  The paper names regex-specific work reduction such as literal
// matching as orthogonal and compatible.  One streaming pass over
// the input (rx_prefilter_run, rx_device.cuh) finds, for every 1 KiB block,
// which regex *factors* occur in it; the interleaved pass then runs a regex's
// cluster in a window only if one of its factors occurs in the window's frame
// (or state forces it, below).
//
// A factor is a window of up to 16 fixed-offset byte positions of the regex
// (exact bytes, one-bit classes such as [Ss], or "any byte"), found in the
// input by its anchor k-gram (hashing) and then compared as a whole.  The long
// window makes factors selective even when the anchor is a common word
// ("HTTP/1.union" rather than "TTP/").
//
// Two kinds ("Mode B"):
//  * first factors, from the bounded prefix of the regex before its first
//    unbounded repetition: every partial match that yields output or reaches
//    a state slot (MatchStar carry, while-loop frontier) contains one of them
//    inside the window frame, so "no first factor in the frame and no state
//    in" implies "zero output and zero state out" (mode A skipping is exact);
//  * output factors, from the bounded suffix: one of them ends at most
//    out_delta bytes before every match end, so "no output factor in the
//    frame" implies "zero output" (mode B: the state a window needs is then
//    reconstructed on demand, rx_device.cuh rx_walk_back).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <map>
#include <set>

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
    return std::min(v, 1.0);
  }
};
const Model &model() {
  static Model m;
  return m;
}

constexpr int kWin = 16;          // factor window positions
constexpr double kMinInfo = 14.0; // bits a factor window must carry (between two and three letters)
constexpr double kMinInfoOut = 6.0;   // output factors may be weak: the runtime mode choice rejects them
                                       // where the input holds them often (rx_mode_b, rx_device.cuh)
constexpr double kMinInfoWeak = 9.0;  // first factors: a weak window beats running in every window
constexpr int kMaxDelta = 256;    // output factors: max bytes from the anchor end to the match end

bool has_unbounded(const Ast &a) {
  if (a.kind == AK::Rep && a.hi < 0) return true;
  for (auto &k : a.kids)
    if (has_unbounded(*k)) return true;
  return false;
}

// Matches strings of one fixed length, position p drawn from out[p] (a
// superset for alternations of equal-length alternatives).
bool fixed_seq(const Ast &a, std::vector<ByteSet> &out, size_t cap = 64) {
  switch (a.kind) {
    case AK::Empty: return true;
    case AK::Set:
      if (out.size() >= cap) return false;
      out.push_back(a.set);
      return true;
    case AK::Cat:
      for (auto &k : a.kids)
        if (!fixed_seq(*k, out, cap)) return false;
      return true;
    case AK::Rep: {
      if (a.hi != a.lo) return false;
      std::vector<ByteSet> one;
      if (!fixed_seq(*a.kids[0], one, cap)) return false;
      if (one.size() * (size_t)a.lo + out.size() > cap) return false;
      for (int i = 0; i < a.lo; ++i) out.insert(out.end(), one.begin(), one.end());
      return true;
    }
    case AK::Alt: {
      std::vector<ByteSet> u;
      bool first = true;
      for (auto &k : a.kids) {
        std::vector<ByteSet> s;
        if (!fixed_seq(*k, s, cap)) return false;
        if (first) {
          u = s;
          first = false;
        } else {
          if (s.size() != u.size()) return false;
          for (size_t i = 0; i < s.size(); ++i) u[i].merge(s[i]);
        }
      }
      if (u.size() + out.size() > cap) return false;
      out.insert(out.end(), u.begin(), u.end());
      return true;
    }
  }
  return false;
}

// longest match length, -1 = unbounded
int max_len(const Ast &a) {
  switch (a.kind) {
    case AK::Empty: return 0;
    case AK::Set: return 1;
    case AK::Cat: {
      long s = 0;
      for (auto &k : a.kids) {
        int m = max_len(*k);
        if (m < 0) return -1;
        s += m;
      }
      return s > (1 << 20) ? -1 : (int)s;
    }
    case AK::Alt: {
      int m = 0;
      for (auto &k : a.kids) {
        int x = max_len(*k);
        if (x < 0) return -1;
        m = std::max(m, x);
      }
      return m;
    }
    case AK::Rep: {
      int m = max_len(*a.kids[0]);
      if (m == 0) return 0;
      if (m < 0 || a.hi < 0) return -1;
      long s = (long)m * a.hi;
      return s > (1 << 20) ? -1 : (int)s;
    }
  }
  return -1;
}

// information (bits) a window position contributes to the extension compare:
// exact bytes and one-bit classes are compared, wider classes are wildcards
double pos_info(const ByteSet &s) {
  const int c = s.count();
  if (c == 0 || c > 2) return 0.0;
  if (c == 2) {
    int b0 = -1, b1 = -1;
    for (int b = 0; b < 256; ++b)
      if (s.has(b)) (b0 < 0 ? b0 : b1) = b;
    if (__builtin_popcount((unsigned)(b0 ^ b1)) != 1) return 0.0;
  }
  return -std::log2(model().set_p(s));
}

bool anchorable(const std::vector<ByteSet> &w) {
  for (size_t i = 0; i + 2 <= w.size(); ++i)
    if ((size_t)w[i].count() * (size_t)w[i + 1].count() <= 256 && w[i].count() > 0 && w[i + 1].count() > 0) return true;
  return false;
}

// best window (<= kWin positions) of a run; returns its start (or -1)
int best_window(const std::vector<ByteSet> &run, double &info) {
  int best = -1;
  info = 0;
  const int n = (int)run.size();
  for (int i = 0; i < n; ++i) {
    const int L = std::min(kWin, n - i);
    double v = 0;
    for (int j = 0; j < L; ++j) v += pos_info(run[i + j]);
    if (v <= info + 1e-9) continue;
    std::vector<ByteSet> w(run.begin() + i, run.begin() + i + L);
    if (!anchorable(w)) continue;
    info = v;
    best = i;
  }
  return best;
}

bool good_run(const std::vector<ByteSet> &run, double min_info = kMinInfo) {
  double info;
  return best_window(run, info) >= 0 && info >= min_info;
}

// ---- first factors: forward over the bounded prefix ------------------------
struct Fwd {
  struct Br {
    std::vector<std::vector<ByteSet>> runs;
    std::vector<ByteSet> cur;
  };
  std::vector<Br> br = std::vector<Br>(1);
  bool stop = false;
  void brk() {
    for (auto &b : br) {
      if (!b.cur.empty()) b.runs.push_back(b.cur);
      b.cur.clear();
    }
  }
  // alternatives of fixed sequences branch the path (<= 8 branches):
  // (GET|POST)xyz -> GETxyz | POSTxyz
  bool branch(const Ast &a) {
    if (a.kind != AK::Alt || has_unbounded(a)) return false;
    std::vector<std::vector<ByteSet>> alts;
    for (auto &k : a.kids) {
      std::vector<ByteSet> s;
      if (!fixed_seq(*k, s)) return false;
      alts.push_back(s);
    }
    if (br.size() * alts.size() > 8) return false;
    std::vector<Br> nb;
    for (auto &b : br)
      for (auto &s : alts) {
        Br x = b;
        x.cur.insert(x.cur.end(), s.begin(), s.end());
        nb.push_back(x);
      }
    br.swap(nb);
    return true;
  }
  void item(const Ast &a) {
    if (stop) return;
    if (branch(a)) return;
    std::vector<ByteSet> fs;
    if (a.kind != AK::Cat && fixed_seq(a, fs)) {  // (a Cat is walked item by item: its alternations may branch)
      for (auto &b : br) b.cur.insert(b.cur.end(), fs.begin(), fs.end());
      return;
    }
    switch (a.kind) {
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
        brk();
        if (has_unbounded(a)) stop = true;
        return;
      default:
        brk();
        return;
    }
  }
};

// best window of each branch; false if some branch has none
bool first_windows(const Ast &a, std::vector<std::vector<ByteSet>> &wins) {
  if (a.kind == AK::Alt) {  // a top-level alternation: the union of its alternatives' factors
    for (auto &k : a.kids)
      if (!first_windows(*k, wins)) return false;
    return !wins.empty();
  }
  Fwd f;
  f.item(a);
  f.brk();
  for (auto &b : f.br) {
    double best_info = 0;
    std::vector<ByteSet> bw;
    for (auto &run : b.runs) {
      double info;
      const int i = best_window(run, info);
      if (i >= 0 && info > best_info) {
        best_info = info;
        bw.assign(run.begin() + i, run.begin() + std::min<size_t>(run.size(), (size_t)i + kWin));
      }
    }
    if (best_info < kMinInfoWeak) return false;
    wins.push_back(bw);
  }
  return true;
}

// ---- output factors: backward over the bounded suffix ----------------------
// emits (run, dist): the run's last position lies `dist` bytes before the
// match end (dist = 0: it is the match end).  Every non-empty match ends with
// one emitted run followed by <= dist bytes.
struct Bwd {
  std::vector<std::pair<std::vector<ByteSet>, int>> emits;
  bool any(const Ast &a, int dist, int depth) {
    if (dist > kMaxDelta || depth > 12) return false;
    std::vector<ByteSet> fs;
    if (a.kind != AK::Alt && fixed_seq(a, fs)) {
      if (good_run(fs, kMinInfoOut)) {
        emits.push_back({fs, dist});
        return true;
      }
      return false;
    }
    switch (a.kind) {
      case AK::Cat: {
        std::vector<const Ast *> it;
        for (auto &k : a.kids) it.push_back(k.get());
        return cat(it, dist, depth);
      }
      case AK::Alt:
        for (auto &k : a.kids) {
          if (k->kind == AK::Empty) continue;  // produces no (non-empty) match end
          if (!any(*k, dist, depth + 1)) return false;
        }
        return true;
      case AK::Rep:  // the last (non-empty) repetition ends the match
        if (a.hi == 0) return true;
        return any(*a.kids[0], dist, depth + 1);
      default:
        return false;
    }
  }
  bool cat(const std::vector<const Ast *> &items, int dist, int depth) {
    std::vector<ByteSet> R;
    // a weak (but anchorable) mandatory run passed on the way: the fallback
    // if nothing strong is found
    std::vector<ByteSet> weak;
    int weak_dist = 0;
    auto keep_weak = [&]() {
      if (weak.empty() && good_run(R, kMinInfoOut)) {
        weak = R;
        weak_dist = dist;
      }
    };
    auto fail = [&]() {
      if (weak.empty()) return false;
      emits.push_back({weak, weak_dist});
      return true;
    };
    for (int i = (int)items.size() - 1; i >= 0; --i) {
      const Ast &it = *items[i];
      std::vector<ByteSet> fs;
      if (fixed_seq(it, fs)) {
        R.insert(R.begin(), fs.begin(), fs.end());
        continue;
      }
      if (good_run(R)) {
        emits.push_back({R, dist});
        return true;
      }
      keep_weak();
      const int d2 = dist + (int)R.size();
      const int ml = max_len(it);
      if (ml >= 0) {
        // a bounded item of variable length: its own factors if it cannot be
        // empty, else a gap of <= ml bytes
        if (!ast_nullable(it)) {
          const size_t mark = emits.size();
          if (any(it, d2, depth + 1)) return true;
          emits.resize(mark);
        }
        dist = d2 + ml;
        R.clear();
        if (dist > kMaxDelta) return fail();
        continue;
      }
      // unbounded: the match ends inside its last repetition, or -- if it can
      // be empty -- right after the items before it
      const size_t mark = emits.size();
      if (!any(it, d2, depth + 1)) {
        emits.resize(mark);
        return fail();
      }
      if (!ast_nullable(it)) return true;
      if (!weak.empty()) {  // the weak run lies after the item: it is in every match
        emits.resize(mark);
        emits.push_back({weak, weak_dist});
        return true;
      }
      dist = d2;
      R.clear();
    }
    if (good_run(R, kMinInfoOut)) {
      emits.push_back({R, dist});
      return true;
    }
    return fail();
  }
};

int add_factor(std::vector<Factor> &table, std::map<std::vector<std::vector<uint64_t>>, int> &ix,
               const std::vector<ByteSet> &win) {  // deduplicated by window
  std::vector<std::vector<uint64_t>> key;
  for (auto &s : win) key.push_back(std::vector<uint64_t>(s.w, s.w + 4));
  auto it = ix.find(key);
  if (it != ix.end()) return it->second;
  Factor f;
  f.win = win;
  double lp = 0;
  for (auto &s : win) lp += std::log(std::max(1e-300, model().set_p(s)));
  f.score = std::exp(lp);
  table.push_back(f);
  const int id = (int)table.size() - 1;
  ix[key] = id;
  return id;
}

}  // namespace

void regex_factors(const Ast &a, CompiledSet &cs, RegexFactors &rf) {
  std::vector<Factor> &table = cs.factors;
  auto &ix = cs.factor_ix;
  rf = RegexFactors();
  std::vector<std::vector<ByteSet>> wins;
  if (first_windows(a, wins) && wins.size() <= 16) {
    std::set<int> ids;
    for (auto &w : wins) ids.insert(add_factor(table, ix, w));
    rf.first.assign(ids.begin(), ids.end());
  }
  Bwd b;
  if (b.any(a, 0, 0) && !b.emits.empty() && b.emits.size() <= 16) {
    std::set<int> ids;
    int delta = 0;
    for (auto &e : b.emits) {
      double info;
      const int i = best_window(e.first, info);
      if (i < 0) return;
      std::vector<ByteSet> w(e.first.begin() + i, e.first.begin() + std::min<size_t>(e.first.size(), (size_t)i + kWin));
      ids.insert(add_factor(table, ix, w));
      // the anchor ends at or after the window's first position
      delta = std::max(delta, e.second + (int)e.first.size() - 1 - i);
    }
    if (delta <= kMaxDelta) {
      rf.out.assign(ids.begin(), ids.end());
      rf.out_delta = delta;
    }
  }
}

// ---------------------------------------------------------------------------
// Device tables of the prefilter, one u32 blob (read by rx_prefilter_run):
//   [0, W4)         Bloom filter over the 4-gram anchors: bit (x * 0x9E3779B1) >> (32 - b4bits)
//   [o_b3, +W3)     Bloom filter over the 3-gram anchors (x >> 8), if any
//   [o_b2, +2048)   bitmap over the 2-gram anchors (x >> 16), if any
//                   (everything before o_ht is staged in shared memory)
//   [o_ht, +4*HS)   open-addressing hash of the anchors: {gram, k << 1 | 1, first ext, n ext}
//   [o_ext, +12*NE) extension entries {ae, xv[4], xm[4], first triple, #triples,
//                   factor}: the window bytes [e - ae, e - ae + 16) of an
//                   anchor ending at e must satisfy (byte & xm) == xv
//   [o_fgoff, nf+1) per factor: its range of {group, member mask, kind} triples
//   [o_fgent, 3*m)  kind 0 = first factor, 1 = output factor
// ---------------------------------------------------------------------------
uint32_t pf_ht_hash(uint32_t gram, uint32_t k) { return (gram ^ (k * 0x27D4EB2Fu)) * 0x9E3779B1u; }

void build_prefilter(CompiledSet &cs) {
  Prefilter &pf = cs.pf;
  pf = Prefilter();
  const int nf = (int)cs.factors.size();
  pf.nfactor = nf;
  const Model &mdl = model();
  // only factors some regex still uses get anchors: output factors are
  // dropped when mode B is off, and an unused anchor would cost filter hits
  // and verification for nothing
  std::vector<char> used(nf, 0);
  for (auto &rf : cs.rf) {
    for (int f : rf.first) used[f] = 1;
    for (int f : rf.out) used[f] = 1;
  }
  // anchors: per factor the rarest k-gram of narrow consecutive positions
  // (k = 4 preferred), spreading factors over distinct anchors (a shared
  // anchor makes every hit verify every factor that uses it)
  std::map<uint32_t, int> uses;
  // how many factor windows contain each exact 4-gram: a gram shared by many
  // rules is likely a protocol keyword that is frequent in traffic too
  // ("HTTP", "Cook"), so anchors avoid it where the window allows
  std::map<uint32_t, int> df;
  auto exact4 = [&](const Factor &F, int j, uint32_t &g) {
    g = 0;
    for (int t = 0; t < 4; ++t) {
      if (F.win[j + t].count() != 1) return false;
      int b0 = 0;
      while (!F.win[j + t].has(b0)) ++b0;
      g = g << 8 | (uint32_t)b0;
    }
    return true;
  };
  for (int f = 0; f < nf; ++f) {
    if (!used[f]) continue;
    std::set<uint32_t> seen;
    for (int j = 0; j + 4 <= (int)cs.factors[f].win.size(); ++j) {
      uint32_t g;
      if (exact4(cs.factors[f], j, g) && seen.insert(g).second) df[g]++;
    }
  }
  auto df_at = [&](const Factor &F, int j, int k) {  // max df over the 4-grams overlapping the anchor
    int m = 1;
    for (int a = std::max(0, j + k - 4); a <= j && a + 4 <= (int)F.win.size(); ++a) {
      uint32_t g;
      if (exact4(F, a, g)) m = std::max(m, df[g]);
    }
    return m;
  };
  for (int f = 0; f < nf; ++f) {
    Factor &F = cs.factors[f];
    F.grams.clear();
    if (!used[f]) continue;  // no anchor, no extension entry
    const int L = (int)F.win.size();
    int bk = 0, bj = -1;
    double bs = 1e300;
    for (int k = 4; k >= 2 && bj < 0; --k) {
      const size_t cap = k == 2 ? 256 : 64;
      for (int j = 0; j + k <= L; ++j) {
        size_t prod = 1;
        double p = 1;
        for (int t = 0; t < k; ++t) {
          prod *= (size_t)F.win[j + t].count();
          p *= mdl.set_p(F.win[j + t]);
        }
        if (prod == 0 || prod > cap) continue;
        // key of the anchor for the diversity penalty: its first gram
        uint32_t key = (uint32_t)k;
        for (int t = 0; t < k; ++t) {
          int b0 = 0;
          while (!F.win[j + t].has(b0)) ++b0;
          key = key * 0x01000193u ^ (uint32_t)b0;
        }
        // a shared anchor makes each of its hits verify every factor using it:
        // strongly prefer anchors no other factor uses
        const double sc = p * std::pow(64.0, (double)uses[key]) * std::pow(32.0, (double)(df_at(F, j, k) - 1));
        if (sc < bs) {
          bs = sc;
          bj = j;
          bk = k;
        }
      }
    }
    if (bj < 0) {  // cannot happen: windows are anchorable by construction
      bj = 0;
      bk = 2;
    }
    {
      uint32_t key = (uint32_t)bk;
      for (int t = 0; t < bk; ++t) {
        int b0 = 0;
        while (!F.win[bj + t].has(b0)) ++b0;
        key = key * 0x01000193u ^ (uint32_t)b0;
      }
      uses[key]++;
    }
    F.ae = bj + bk - 1;
    // enumerate the anchor grams: byte t of the gram at bit 8*(4-k+t)
    std::vector<FactorGram> g(1, FactorGram{0u, 0u, bk});
    for (int t = 0; t < bk; ++t) {
      std::vector<FactorGram> ng;
      for (int b = 0; b < 256; ++b)
        if (F.win[bj + t].has(b))
          for (auto &x : g) ng.push_back(FactorGram{x.gram | ((uint32_t)b << (8 * (4 - bk + t))), 0u, bk});
      g.swap(ng);
    }
    const uint32_t mask = bk == 4 ? 0xffffffffu : (0xffffffffu << (8 * (4 - bk)));
    for (auto &x : g) x.mask = mask;
    F.grams = g;
    // extension compare
    for (int t = 0; t < 16; ++t) {
      F.xv[t] = F.xm[t] = 0;
      if (t >= L) continue;
      const ByteSet &s = F.win[t];
      const int c = s.count();
      int b0 = -1, b1 = -1;
      for (int b = 0; b < 256; ++b)
        if (s.has(b)) (b0 < 0 ? b0 : b1) = b;
      if (c == 1) {
        F.xm[t] = 0xff;
        F.xv[t] = (uint8_t)b0;
      } else if (c == 2 && __builtin_popcount((unsigned)(b0 ^ b1)) == 1) {
        F.xm[t] = (uint8_t)(0xff & ~(b0 ^ b1));
        F.xv[t] = (uint8_t)(b0 & F.xm[t]);
      }
    }
  }
  // anchor -> extension entries
  std::map<std::pair<uint32_t, int>, std::vector<int>> slots;  // (gram, k) -> factors
  int n4 = 0, n3 = 0, n2 = 0;
  for (int f = 0; f < nf; ++f)
    for (auto &g : cs.factors[f].grams) {
      auto &v = slots[{g.gram, g.k}];
      if (v.empty()) (g.k == 4 ? n4 : (g.k == 3 ? n3 : n2))++;
      v.push_back(f);
    }
  auto lg = [](int n, int lo, int hi) {
    int b = lo;
    while (b < hi && (1 << b) < n * 128) ++b;
    return b;
  };
  pf.b4bits = (uint32_t)lg(std::max(n4, 1), 13, 18);
  const uint32_t b3bits = (uint32_t)lg(std::max(n3, 1), 10, 16);
  std::vector<uint32_t> &B = pf.blob;
  B.assign((size_t)1 << (pf.b4bits - 5), 0u);
  std::vector<uint32_t> bl3(n3 ? (size_t)1 << (b3bits - 5) : 0, 0u), bg2(n2 ? 2048 : 0, 0u);
  for (auto &kv : slots) {
    const uint32_t gram = kv.first.first;
    const int k = kv.first.second;
    if (k == 4) {
      const uint32_t h = (gram * 0x9E3779B1u) >> (32 - pf.b4bits);
      B[h >> 5] |= 1u << (h & 31);
    } else if (k == 3) {
      const uint32_t h = ((gram >> 8) * 0x85EBCA77u) >> (32 - b3bits);
      bl3[h >> 5] |= 1u << (h & 31);
    } else {
      const uint32_t h = gram >> 16;
      bg2[h >> 5] |= 1u << (h & 31);
    }
  }
  if (n3) {
    pf.o_b3 = (uint32_t)B.size();
    B.insert(B.end(), bl3.begin(), bl3.end());
  }
  if (n2) {
    pf.o_b2 = (uint32_t)B.size();
    B.insert(B.end(), bg2.begin(), bg2.end());
  }
  // factor -> (group, member mask, kind); kind 0 = first factor, 1 = output factor
  std::vector<std::map<std::pair<int, int>, uint32_t>> fg(nf);
  for (int gi = 0; gi < (int)cs.groups.size(); ++gi) {
    const Group &g = cs.groups[gi];
    for (size_t m = 0; m < g.regexes.size(); ++m) {
      const RegexFactors &rf = cs.rf[g.regexes[m]];
      for (int f : rf.first) fg[f][{gi, 0}] |= 1u << m;
      for (int f : rf.out) fg[f][{gi, 1}] |= 1u << m;
    }
  }
  std::vector<uint32_t> fgoff, fge;
  for (int f = 0; f < nf; ++f) {
    fgoff.push_back((uint32_t)(fge.size() / 3));
    for (auto &kv : fg[f]) fge.insert(fge.end(), {(uint32_t)kv.first.first, kv.second, (uint32_t)kv.first.second});
  }
  fgoff.push_back((uint32_t)(fge.size() / 3));
  pf.smem_words = (uint32_t)B.size();
  pf.o_ht = (uint32_t)B.size();
  uint32_t hs = 64;
  while (hs < 2 * slots.size()) hs <<= 1;
  pf.hbits = 0;
  while ((1u << pf.hbits) < hs) ++pf.hbits;
  std::vector<uint32_t> ht(4 * (size_t)hs, 0u), ext;
  for (auto &kv : slots) {
    const uint32_t gram = kv.first.first, k = (uint32_t)kv.first.second;
    uint32_t h = pf_ht_hash(gram, k) >> (32 - pf.hbits);
    while (ht[4 * h + 1] != 0u) h = (h + 1) & (hs - 1);
    ht[4 * h] = gram;
    ht[4 * h + 1] = (k << 1) | 1u;
    ht[4 * h + 2] = (uint32_t)(ext.size() / 12);
    ht[4 * h + 3] = (uint32_t)kv.second.size();
    for (int f : kv.second) {
      const Factor &F = cs.factors[f];
      ext.push_back((uint32_t)F.ae);
      for (int w = 0; w < 4; ++w)
        ext.push_back((uint32_t)F.xv[4 * w] | (uint32_t)F.xv[4 * w + 1] << 8 | (uint32_t)F.xv[4 * w + 2] << 16 |
                      (uint32_t)F.xv[4 * w + 3] << 24);
      for (int w = 0; w < 4; ++w)
        ext.push_back((uint32_t)F.xm[4 * w] | (uint32_t)F.xm[4 * w + 1] << 8 | (uint32_t)F.xm[4 * w + 2] << 16 |
                      (uint32_t)F.xm[4 * w + 3] << 24);
      ext.push_back(fgoff[f]);
      ext.push_back(fgoff[f + 1] - fgoff[f]);
      ext.push_back((uint32_t)f);
    }
  }
  B.insert(B.end(), ht.begin(), ht.end());
  pf.o_ext = (uint32_t)B.size();
  B.insert(B.end(), ext.begin(), ext.end());
  // factor -> (group, member mask, kind) triples, referenced from the
  // extension entries directly (one dependent load less per verified hit)
  pf.o_fgoff = (uint32_t)B.size();
  pf.o_fgent = pf.o_fgoff + (uint32_t)fgoff.size();
  B.insert(B.end(), fgoff.begin(), fgoff.end());
  B.insert(B.end(), fge.begin(), fge.end());
  // remember b3bits next to hbits: hbits | b3bits << 8
  pf.hbits |= b3bits << 8;
}

std::string factor_info(const CompiledSet &cs, int r) {
  auto win = [&](int f) {
    const Factor &F = cs.factors[f];
    std::string s;
    char b[8];
    for (size_t t = 0; t < F.win.size() && t < 16; ++t) {
      snprintf(b, sizeof b, "%02x%02x", F.xv[t], F.xm[t]);
      s += b;
    }
    snprintf(b, sizeof b, "@%d/%d", F.ae, F.grams.empty() ? 0 : F.grams[0].k);
    return s + b;
  };
  std::string o = "first";
  const RegexFactors &rf = cs.rf[r];
  if (rf.first.empty()) o += " none";
  for (int f : rf.first) o += " " + win(f);
  o += " ; out";
  if (rf.out.empty()) o += " none";
  for (int f : rf.out) o += " " + win(f);
  o += " ; delta=" + std::to_string(rf.out_delta);
  return o;
}

}  // namespace rx
