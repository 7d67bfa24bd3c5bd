// rx_internal.h -- host compiler internals: AST, bitstream IR, groups.
//
// PAPER.md references (P:Lnnn): grammar P:L67-69 (Listing 1 lost);
// lowering rules Fig. 2 and Listing 3; bitstream
// program grammar P:L118 (Listing 2 lost).
#pragma once
#include <cstdint>
#include <map>
#include <memory>
#include <string>
#include <vector>

namespace rx {

// 256-bit byte set.
struct ByteSet {
  uint64_t w[4] = {0, 0, 0, 0};
  void set(int c) { w[c >> 6] |= 1ull << (c & 63); }
  bool has(int c) const { return (w[c >> 6] >> (c & 63)) & 1; }
  void range(int a, int b) { for (int c = a; c <= b; ++c) set(c); }
  void invert() { for (auto &x : w) x = ~x; }
  void merge(const ByteSet &o) { for (int i = 0; i < 4; ++i) w[i] |= o.w[i]; }
  bool empty() const { return !(w[0] | w[1] | w[2] | w[3]); }
  bool full() const { return !~(w[0] & w[1] & w[2] & w[3]); }
  int count() const { int n = 0; for (auto x : w) n += __builtin_popcountll(x); return n; }
  bool operator==(const ByteSet &o) const { return w[0] == o.w[0] && w[1] == o.w[1] && w[2] == o.w[2] && w[3] == o.w[3]; }
};

// ----------------------------------------------------------------------------
// AST (the compiler's own parser; the oracle has a separate one)
// ----------------------------------------------------------------------------
enum class AK : uint8_t { Empty, Set, Cat, Alt, Rep };
struct Ast {
  AK kind = AK::Empty;
  ByteSet set;                       // Set
  std::vector<std::unique_ptr<Ast>> kids;  // Cat / Alt: items; Rep: kids[0]
  int lo = 0, hi = 0;                // Rep: hi < 0 = unbounded
};
using AstP = std::unique_ptr<Ast>;

struct ParseError {
  int code;  // rx_status: 1 parse, 2 unsupported, 3 too big
  size_t at;
  std::string msg;
};

// Returns nullptr and fills err on failure.
AstP parse_regex(const std::string &pat, ParseError &err);
bool ast_nullable(const Ast &a);
size_t ast_expanded_size(const Ast &a);  // #Set leaves after R{n,m} expansion (for caps)

// ----------------------------------------------------------------------------
// Bitstream IR (per regex).  Streams are indexed by input position p (bit p of
// word p/32, LSB-first; SURVEY App.A-1).  Paper's "S >> k" (advance) = Adv.
// ----------------------------------------------------------------------------
enum class Op : uint8_t {
  Zero,    // all-zero stream
  Ones,    // all-ones stream incl. positions < 0 (the unanchored start marker, DESIGN "start")
  CC,      // character class from the basis streams (Fig. 2a)
  And, Or, Xor, AndNot,  // AndNot(a,b) = a & ~b
  Adv,     // out[p] = in[p-k]  (paper ">> k", Fig. 2b); inside loop bodies: forwarded site
  Look,    // out[p] = in[p+k]  (paper "<< k", produced by Shift Rebalancing)
  MStar,   // ends of X C*: ((((X + C) ^ C) | X) & C), X subset C (MatchStar, Parabix [24])
  Loop,    // while-fixpoint of Fig. 2e / Listing 3: acc = lfp(seeds U body(acc))
  Fr,      // the frontier placeholder inside a Loop body
  Guard,   // zero-block-skipping region (Sec. 6): value = region result, or 0 if any(cond)==0
  Lit,     // literal run: out[p] = in[p-k] & (input[p-k+1..p] == lits[cc]) -- exactly the chain
           // v_j = Adv(v_{j-1}, 1) & CC(lits[cc][j]) (Fig. 2b/2c) for j = 1..k, evaluated by
           // confirming the (sparse) marker positions byte by byte
};

struct Node {
  Op op = Op::Zero;
  int a = -1, b = -1;  // operands (node ids); Guard: a = condition; Loop: a = seeds
  int k = 0;           // Adv / Look distance
  int cc = -1;         // CC: index into Program::sets
  int sub = -1;        // Loop / Guard: body block id
  int res = -1;        // Loop: body result E(R, Fr); Guard: region result
  int fr = -1;         // Loop: its Fr node
  int loop = -1;       // innermost enclosing Loop node (-1: top level)
  // analysis
  int lb = 0, rb = 0;  // invalid bits at the window's left / right edge (margins, DESIGN "Margins")
  int aw = 0;          // stateful: injection word (MStar, forwarded Adv, Loop)
  int slot = -1;       // stateful: state slot (MStar carry, forwarded Adv tail)
  int depth = 0;       // longest op path from inputs (Shift Rebalancing)
};

struct Block {
  std::vector<int> nodes;  // emission order
};

struct RegexIR {
  std::vector<Node> nodes;
  std::vector<Block> blocks;  // blocks[0] = top level
  std::vector<ByteSet> sets;
  std::vector<std::string> lits;  // Lit: literal byte strings (no 0x00 byte)
  int out = -1;               // result node (top level) of a single-regex IR
  std::vector<int> outs;      // result nodes of a cluster IR (one per member regex; outs[0] == out)
  int nslots = 0;
  int lb = 0, rb = 0;         // margins of the output (bits)
  int rb_state = 0;           // max rb over inputs of stateful sites (bits)
  size_t n_instr = 0;         // instruction count (for grouping / guards)
  int n_loops = 0, n_mstar = 0, n_adv = 0, n_guards = 0;
};

struct LowerOptions {
  int interval = 8;       // guard interval (instructions), <= 0: no guards
  bool rebalance = true;
  // no zero-block guard inside the leading run of single-class items of an
  // unanchored chain (with the prefilter the regex only runs where its
  // factor occurs, and an unguarded head can be shared by a factor cluster)
  bool lead_noguard = false;
  // literal runs: after `lit_after` single-byte items of a chain (the marker
  // stream is then sparse), a run of >= lit_min further single-byte items
  // becomes one Lit node; lit_min <= 0: never
  int lit_after = 3;
  int lit_min = 2;
};

// Lower one parsed regex to IR (non-empty, unanchored match ends).
void lower_regex(const Ast &ast, const LowerOptions &opt, RegexIR &ir);
// Lower several regexes into one IR with shared (hash-consed) nodes: a
// factor cluster of a group is evaluated once per window (DESIGN.md
// "Clusters").  ir.outs[i] is the result of asts[i].
void lower_cluster(const std::vector<const Ast *> &asts, const LowerOptions &opt, RegexIR &ir);
// Shift Rebalancing (Sec. 5.2): operand rewriting to a fixpoint + merging.
void rebalance_regex(RegexIR &ir);
// Compute margins, injection words and state slots.  Returns false if a
// construct is not representable (message in why).
bool analyze_regex(RegexIR &ir, std::string &why);
std::string dump_ir(const RegexIR &ir);

// ----------------------------------------------------------------------------
// Groups and program geometry
// ----------------------------------------------------------------------------
struct Cluster {
  std::vector<int> members;  // member indices (into Group::regexes), in IR output order
  RegexIR ir;                // shared IR of the members (lower_cluster)
  int slot_base = 0;         // first state slot of the cluster in the group
  bool always = false;       // members without a factor: runs in every window
  bool bcap = false;         // every member has output factors: may run output-gated (mode B)
};

struct Group {
  std::vector<int> regexes;  // global regex ids
  uint32_t always = 0;       // members without a prefilter factor (run in every window)
  std::vector<Cluster> clusters;  // the group's code: members sharing a factor evaluated together
  int K = 1;                 // words per lane per window
  int Lw = 0, Rw = 0, Bw = 0;  // window: left halo words, right halo words, committed words (32K = Lw+Bw+Rw)
  int nslots = 0;
  std::vector<int> slot_base;  // per member regex
  double cost = 0;
  int out_delta = 0;         // max output-factor distance of a member (bytes; the halo covers it)
};

// Cross-regex literal prefilter (rx_prefilter.cpp).
// A factor is a window of up to 16 fixed-offset byte positions that every
// (partial) match must contain: each position is an exact byte, a byte up to
// one bit (e.g. [Ss]), or any byte.  Its *anchor* is a k-gram (2 <= k <= 4)
// of consecutive narrow positions inside the window, found by hashing; the
// whole window is then compared.
struct FactorGram {
  uint32_t gram, mask;  // bytes of the k-gram in the top k bytes of a little-endian u32 window
  int k;
  bool operator==(const FactorGram &o) const { return gram == o.gram && mask == o.mask; }
};
struct Factor {
  std::vector<ByteSet> win;       // the window's positions (<= 16)
  std::vector<FactorGram> grams;  // anchor alternatives (chosen by build_prefilter)
  int ae = 0;                     // window index of the anchor's last byte
  uint8_t xv[16] = {0}, xm[16] = {0};  // window bytes [e - ae, e - ae + 16): (byte & xm) == xv
  double score = 0;               // estimated occurrences per position (ranking only)
};
struct Prefilter {
  int nfactor = 0;
  std::vector<uint32_t> blob;  // device table layout: see rx_prefilter_run (rx_device.cuh)
  uint32_t b4bits = 0;         // log2 bits of the 4-gram Bloom filter
  uint32_t o_b3 = 0, o_b2 = 0; // word offsets of the 3-gram Bloom / bigram bitmap (0 = none)
  uint32_t o_ht = 0, hbits = 0;  // anchor hash table {gram, k<<1|1, first ext, n ext}, log2 slots
  uint32_t o_ext = 0;          // extension entries {ae, v[4], m[4], fid}
  uint32_t o_fgoff = 0, o_fgent = 0;  // factor -> {group, member mask, kind} triples
  uint32_t smem_words = 0;     // leading words staged in shared memory (Bloom filters + bitmap)
};
// Per-regex factors.  first: prefix factors -- one of them lies inside every
// partial match that produces output or reaches a state slot (empty: the
// regex runs in every window).  out: output factors -- one of them ends at
// most out_delta bytes before every match end (empty: none; the regex then
// cannot run in output-gated mode B).
struct RegexFactors {
  std::vector<int> first, out;
  int out_delta = 0;
};

struct CompiledSet {
  int pass1_warps = 16;           // warps per pass-1 CTA (rx_runtime.cpp rx_compile)
  std::vector<int> factor_of;     // per regex: clustering key of its first-factor set, -1 = none (always runs)
  std::vector<RegexFactors> rf;   // per regex
  std::vector<Factor> factors;
  std::map<std::vector<std::vector<uint64_t>>, int> factor_ix;  // factor window -> id (deduplication)
  Prefilter pf;
  bool use_pf = false;
  std::vector<RegexIR> irs;
  std::vector<Group> groups;
  std::string source;  // generated CUDA C
  std::string info;
};

// First and output factors of one regex, added to cs.factors (deduplicated).
void regex_factors(const Ast &a, CompiledSet &cs, RegexFactors &rf);

// CUDA C sources: one relocatable unit per group + the kernel unit; linked
// into one module with nvJitLink.
std::string emit_group_unit(CompiledSet &cs, int gi);
std::string emit_kernel_unit(CompiledSet &cs, int gb, int ge);  // kernels of module [gb, ge)
int lit_scratch_bytes(const CompiledSet &cs);  // per-warp shared bytes of the literal-run scratch
int max_words_per_lane(const CompiledSet &cs);
size_t warp_smem_bytes(const CompiledSet &cs);  // per-warp shared bytes of pass 1 / fix-up
bool plan_groups(CompiledSet &cs, int group_size, int force_K, std::string &why);
void build_prefilter(CompiledSet &cs);
std::string factor_info(const CompiledSet &cs, int r);  // "first [...] out [...]" (rx_program_info)
// Partition each group's members into clusters (same factor, or no factor)
// and lower each cluster jointly; recomputes the group's state slots.
bool build_clusters(CompiledSet &cs, const std::vector<const Ast *> &asts, const LowerOptions &opt,
                    std::string &why);

}  // namespace rx
