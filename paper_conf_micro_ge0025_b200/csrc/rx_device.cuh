// rx_device.cuh -- hand-written sm_100a device template of the fused
// interleaved bitstream kernel (Sec. 3.3: "all
// bitstream instructions are fused into a single loop ... executed
// block-wise").  NVRTC compiles this together with the generated program
// bodies (rx_codegen.cpp).  No #includes: NVRTC-only builtins.
//
// B200 design:
//  * one WARP runs one regex group over a contiguous segment of windows; a
//    window is 32 lanes x K words x 32 positions (lane-major: lane l holds
//    words [lK, lK+K)); cross-word shifts are funnel shifts plus one
//    __shfl per K words -- no shared-memory staging and no CTA barriers
//    (the paper's per-SHIFT barrier pairs, vanish at warp scope);
//  * static shifts are resolved by recomputing a halo of Lw/Rw words
//    (Dependency-Aware Thread-Data Mapping, Sec. 4.2, with
//    per-side margins, SURVEY App.A-8);
//  * unbounded dependencies (MatchStar carries, while-loop frontiers) are
//    carried across windows as uniform state words injected at a fixed word
//    -- exact with no overflow limit (the paper's P:L503 limitation);
//  * the byte->basis transposition is fused into the window
//    prologue: 128-bit loads, a 16-PRMT byte transpose and a 3-stage SWAR
//    bit transpose per 32 bytes;
//  * zero-block skipping uses __any_sync votes (warp-uniform branches, the
//    paper's block-wide atomicOr of P:L372 at warp scope);
//  * the epilogue popcounts committed words (REDUX), folds positions into
//    additive digests and optionally stores the dense match bitstreams.
typedef unsigned int u32;
typedef unsigned long long u64;
typedef long long i64;
#define DEV __device__ __forceinline__
#define RX_FULL 0xffffffffu
#define RX_LOOP_CAP (1u << 22)

template <int K>
struct V {
  u32 w[K];
};

DEV u32 rx_lane() {
  u32 l;
  asm volatile("mov.u32 %0, %%laneid;" : "=r"(l));
  return l;
}

// ---------------------------------------------------------------------------
// window context (scalars only: the 8 basis streams live in a register array
// of the segment loop and are passed to the body separately)
// ---------------------------------------------------------------------------
template <int K>
struct Ctx {
  u32 vm[K];    // positions holding real stream bytes
  u32 cm[K];    // committed positions of this window inside [0, len)
  u32 lane;
  u32 cw;       // committed words of this window
  u64 *acc;     // per-warp shared accumulators [NR][3] (count, d1, d2)
  u32 *dense;   // nullable
  u64 pitch;
  i64 word0;    // chunk word index of local word 0
  i64 gofs;     // global position of chunk position 0
  u64 sign;     // 1 (add) or 2^64-1 (subtract; fix-up pass)
  bool want_digest, want_dense;
  const int *rid;  // group member -> global regex id
  u32 *status;
  u64 *mlist;      // nullable: compacted match list, {regex, pos} pairs (rx_match_t)
  u64 mcap;
  u64 *mtotal;
  u32 *fold;       // fix-up only: [NR][K] output words of the "old" run (match-list delta)
  unsigned char *wb;  // nullable (groups without literal runs): the frame's bytes, frame position f at wb[f]
  u32 *ob;            // literal-run output scratch, 32*K words (per warp)
};

// ---------------------------------------------------------------------------
// epilogue (called only when the output has a set bit in the committed
// range, or when dense output is requested): popcount -> REDUX, digests,
// dense store
// ---------------------------------------------------------------------------
DEV u64 rx_splitmix64(u64 x) {
  u64 z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

DEV u64 rx_warp_sum64(u64 v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(RX_FULL, v, o);
  return v;
}

// Compacted match list (rx_output.d_matches): every set bit of the committed
// words becomes one {regex, global position} entry; a warp reserves its slots
// with one atomicAdd and each lane writes its own bits after an exclusive
// prefix sum.  The fix-up's "old" run (sign = -1) records its words in c.fold
// and the "new" run lists only the bits the old one lacked: match sets are
// monotone in the incoming state (every operation on state streams is AND /
// OR / Advance / add-with-carry of a marker into a class), so new covers old;
// a violation is flagged in status bit 2 instead of being silently dropped.
template <int K>
DEV void rx_emit_list(const Ctx<K> &c, int r, const u32 (&m)[K]) {
  u32 mm[K];
  u32 cnt = 0;
  bool lost = false;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    if (c.fold && c.sign == ~0ull) {
      c.fold[r * K + i] = m[i];
      mm[i] = 0u;
    } else if (c.fold) {
      lost = lost || (c.fold[r * K + i] & ~m[i]) != 0u;
      mm[i] = m[i] & ~c.fold[r * K + i];
    } else {
      mm[i] = m[i];
    }
    cnt += __popc(mm[i]);
  }
  if (lost) atomicOr(c.status, 4u);
  u32 incl = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u32 t = __shfl_up_sync(RX_FULL, incl, o);
    if (c.lane >= (u32)o) incl += t;
  }
  const u32 tot = __shfl_sync(RX_FULL, incl, 31);
  if (tot == 0u) return;
  u64 base = 0;
  if (c.lane == 0) base = atomicAdd(c.mtotal, (u64)tot);
  base = __shfl_sync(RX_FULL, base, 0) + (incl - cnt);
  const u64 reg = (u64)(u32)c.rid[r];
#pragma unroll
  for (int i = 0; i < K; ++i) {
    u32 b = mm[i];
    const i64 wpos = c.gofs + (c.word0 + (i64)(c.lane * K + i)) * 32;
    while (b) {
      const int t = __ffs(b) - 1;
      b &= b - 1u;
      if (base < c.mcap) {
        c.mlist[2 * base] = reg;
        c.mlist[2 * base + 1] = (u64)(wpos + t);
      }
      ++base;
    }
  }
}

template <int K>
__device__ __noinline__ void rx_emit(const Ctx<K> c, int r, const V<K> v) {
  u32 m[K];
  u32 any = 0u;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    m[i] = v.w[i] & c.cm[i];
    any |= m[i];
  }
  if (c.want_dense) {
    u32 *row = c.dense + (u64)c.rid[r] * c.pitch;
#pragma unroll
    for (int i = 0; i < K; ++i)
      if (c.cm[i] != 0u) row[c.word0 + (i64)(c.lane * K + i)] = m[i];
  }
  if (!__any_sync(RX_FULL, any != 0u)) return;
  u32 cnt = 0;
#pragma unroll
  for (int i = 0; i < K; ++i) cnt += __popc(m[i]);
  const u32 tot = __reduce_add_sync(RX_FULL, cnt);
  u64 d1 = 0, d2 = 0;
  if (c.want_digest) {
#pragma unroll
    for (int i = 0; i < K; ++i) {
      u32 b = m[i];
      const i64 base = c.gofs + (c.word0 + (i64)(c.lane * K + i)) * 32;
      while (b) {
        const int t = __ffs(b) - 1;
        b &= b - 1u;
        const u64 p = (u64)(base + t);
        d1 += rx_splitmix64(p);
        d2 += rx_splitmix64(p ^ 0x9E3779B97F4A7C15ull);
      }
    }
    d1 = rx_warp_sum64(d1);
    d2 = rx_warp_sum64(d2);
  }
  if (c.lane == 0) {
    c.acc[3 * r + 0] += c.sign * (u64)tot;
    c.acc[3 * r + 1] += c.sign * d1;
    c.acc[3 * r + 2] += c.sign * d2;
  }
  if (c.mtotal) rx_emit_list<K>(c, r, m);
}

// ---------------------------------------------------------------------------
// literal run (IR Op::Lit): out[p] = v[p-n] &
// (bytes p-n+1..p == lit[0..n)), the exact result of the chain
// v_j = Adv(v_{j-1}, 1) & CC(lit[j-1]) (Fig. 2b/2c), evaluated at
// the marker bits only: each lane confirms its own bits against the frame's
// bytes in shared memory and ORs the hits into a per-warp word buffer.
// Output bits beyond the frame fall off, as the advances would shift them
// out; the literal holds no 0x00 byte, so positions outside the stream
// (read as 0) never confirm.
// ---------------------------------------------------------------------------
template <int K>
__device__ __noinline__ V<K> rx_lit(const u32 lane, const unsigned char *wb, u32 *ob, const V<K> v,
                                    const unsigned char *lit, int n) {
  V<K> r;
  u32 any = 0u;
#pragma unroll
  for (int i = 0; i < K; ++i) any |= v.w[i];
  if (!__any_sync(RX_FULL, any != 0u)) {
#pragma unroll
    for (int i = 0; i < K; ++i) r.w[i] = 0u;
    return r;
  }
#pragma unroll
  for (int i = 0; i < K; ++i) ob[lane * K + i] = 0u;
  __syncwarp();
  const int F = 1024 * K;
  const unsigned char l0 = lit[0];
#pragma unroll
  for (int i = 0; i < K; ++i) {
    u32 b = v.w[i];
    while (b) {
      const int t = __ffs(b) - 1;
      b &= b - 1u;
      const int q = (int)((lane * K + i) * 32u) + t;
      const int e = q + n;
      if (e >= F || wb[q + 1] != l0) continue;
      int j = 1;
      while (j < n && wb[q + 1 + j] == lit[j]) ++j;
      if (j == n) atomicOr(&ob[e >> 5], 1u << (e & 31));
    }
  }
  __syncwarp();
#pragma unroll
  for (int i = 0; i < K; ++i) r.w[i] = ob[lane * K + i];
  __syncwarp();
  return r;
}

// ---------------------------------------------------------------------------
// prologue: load + fused transposition
// ---------------------------------------------------------------------------
// 32 bytes x[0..7] (little-endian words) -> 8 basis words: plane[k] bit j =
// bit k of byte j (paper b_{7-k}, b0 = MSB).
DEV void rx_transpose32(const u32 x[8], u32 plane[8]) {
  // byte transpose: y[r] byte q = byte (8q + r)
  u32 y[8];
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const u32 a = x[0 + h], b = x[2 + h], cc = x[4 + h], d = x[6 + h];
    const u32 t0 = __byte_perm(a, b, 0x5140), t1 = __byte_perm(a, b, 0x7362);
    const u32 t2 = __byte_perm(cc, d, 0x5140), t3 = __byte_perm(cc, d, 0x7362);
    y[4 * h + 0] = __byte_perm(t0, t2, 0x5410);
    y[4 * h + 1] = __byte_perm(t0, t2, 0x7632);
    y[4 * h + 2] = __byte_perm(t1, t3, 0x5410);
    y[4 * h + 3] = __byte_perm(t1, t3, 0x7632);
  }
  // 8x8 bit transpose inside each byte lane, across the 8 registers
#define RX_SWAP(r0, r1, s, m)                   \
  {                                             \
    const u32 t = ((y[r0] >> (s)) ^ y[r1]) & (m); \
    y[r1] ^= t;                                 \
    y[r0] ^= t << (s);                          \
  }
  RX_SWAP(0, 4, 4, 0x0F0F0F0Fu) RX_SWAP(1, 5, 4, 0x0F0F0F0Fu) RX_SWAP(2, 6, 4, 0x0F0F0F0Fu) RX_SWAP(3, 7, 4, 0x0F0F0F0Fu)
  RX_SWAP(0, 2, 2, 0x33333333u) RX_SWAP(1, 3, 2, 0x33333333u) RX_SWAP(4, 6, 2, 0x33333333u) RX_SWAP(5, 7, 2, 0x33333333u)
  RX_SWAP(0, 1, 1, 0x55555555u) RX_SWAP(2, 3, 1, 0x55555555u) RX_SWAP(4, 5, 1, 0x55555555u) RX_SWAP(6, 7, 1, 0x55555555u)
#undef RX_SWAP
#pragma unroll
  for (int k = 0; k < 8; ++k) plane[k] = y[k];
}

struct RxParams {
  const unsigned char *in;  // chunk position 0
  i64 avail_lo, avail_hi;   // readable positions
  i64 valid_lo, valid_hi;   // positions holding stream bytes (vm)
  i64 len;                  // committed positions [0, len)
  i64 gofs;                 // global position of chunk position 0
  u64 *counts;
  u64 *digests;
  u32 *dense;
  u64 pitch;
  u32 *status;
  u32 *seg_state;           // [nseg_max][G][NSMAX]
  const u32 *st_in;         // chunk boundary state in (nullable)
  u32 *st_out;              // chunk boundary state out (nullable)
  const u32 *st_assumed;    // rematch: state the chunk was matched with (nullable = zero)
  int sw;                   // windows per segment
  int nseg_max;
  int aligned;              // in is 16-byte aligned
  int mode;                 // 0 = pass 1, 1 = fix-up with stored segment states, 2 = rematch
  int accumulate;           // counts/digests are added to (else the host zeroed them)
  int lockstep;             // pass 1: one CTA barrier per window (warps of a group stay in step)
  // cross-regex prefilter (rx_prefilter below)
  // one table blob (rx_prefilter.cpp build_prefilter), u32 words:
  //   [0,2048) l1 bigram bitmap | [2048,4096) rank: set bits before word i |
  //   bsid[nb]: shapes indexed by each set bigram (shape = 3*(k-2) + d) |
  //   htab[2 << hbits]: {gram, fid << 8 | shape << 1 | 1} | fgoff[nf+1] |
  //   fgent[2*nfe]: {group, member mask}
  const u32 *pf_tab;
  u32 pf_words;             // blob size
  u32 pf_o_ent, pf_o_fgoff, pf_o_fgent;  // word offsets: hash table, factor -> group ranges, pairs
  u32 pf_hbits;             // log2 hash slots
  int pf_tab_smem;          // the whole blob is staged in shared memory
  u32 *pf_gbits;            // [NG][ntiles]: bit b of word t = factor of the group in block 32t+b
  u32 *pf_mmask;            // [NG][32*ntiles]: members of the group whose factor occurs in the block
                            // (written only where non-zero: read only where the pf_gbits bit is set)
  i64 pf_ntiles;
  int pf_on;
  int pf_aligned;           // in + avail_lo is 16-byte aligned
  u64 *stats;               // nullable: debug counters (RX_STATS=1), see rx_run_segment_pf
  int dbg;                  // timing experiments only (RX_DBG): 1 = skip every window, 2 = no body
  u64 *matches;             // nullable: rx_match_t[match_cap] as u64 pairs {regex, pos}
  u64 match_cap;
  u64 *match_total;         // u64: matches found (may exceed match_cap)
  int fix_phase;            // mode 1: 0 = serial fix-up, 1 = parallel per segment, 2 = serial remainder
  u32 *seg_fix;             // [nseg_max][G][NSMAX]: phase-1 end state of a segment that did not converge
  u32 *seg_nc;              // [nseg_max][G]: that segment did not converge in phase 1
  u64 *task_ctr;            // pass 1: non-null = persistent warps pull (group, segment) tasks from it
  int cmajor;               // sparse pass 1 runs cluster by cluster (rx_run_segment_cm)
  int cm_sync;              // ... with one CTA barrier per cluster (static task map only)
};

template <int K> DEV void rx_load_window(const RxParams &p, Ctx<K> &c, u32 (&pl)[8][K], i64 fword) {
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const i64 wi = fword + (i64)(c.lane * K + i);
    const i64 pos = wi * 32;
    u32 x[8];
    if (p.aligned && pos >= p.avail_lo && pos + 32 <= p.avail_hi) {
      const uint4 *q = reinterpret_cast<const uint4 *>(p.in + pos);
      const uint4 a = __ldg(q), b = __ldg(q + 1);
      x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w;
      x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
    } else {
#pragma unroll
      for (int j = 0; j < 8; ++j) x[j] = 0u;
      for (int j = 0; j < 32; ++j) {
        const i64 ps = pos + j;
        if (ps >= p.avail_lo && ps < p.avail_hi) x[j >> 2] |= (u32)p.in[ps] << (8 * (j & 3));
      }
    }
    u32 t[8];
    rx_transpose32(x, t);
#pragma unroll
    for (int k = 0; k < 8; ++k) pl[k][i] = t[k];
    // valid-data mask
    const i64 lo = p.valid_lo - pos, hi = p.valid_hi - pos;  // valid bits [lo, hi) of this word
    u32 m;
    if (lo <= 0 && hi >= 32) m = RX_FULL;
    else if (hi <= 0 || lo >= 32) m = 0u;
    else {
      const u32 a = lo <= 0 ? RX_FULL : (RX_FULL << (u32)lo);
      const u32 b = hi >= 32 ? RX_FULL : (RX_FULL >> (u32)(32 - hi));
      m = a & b;
    }
    c.vm[i] = m;
  }
}

// split prologue (software pipelining): rx_fetch issues the 128-bit loads of
// a window into registers, rx_unpack transposes them one window later.
// Interior windows (all bytes readable and valid, 16-byte aligned) take the
// straight path; edge windows go through an out-of-line byte loader.
struct RxW8 {
  u32 v[8];
};
static __device__ __noinline__ RxW8 rx_fetch_word_slow(const unsigned char *in, i64 avail_lo, i64 avail_hi, i64 pos) {
  RxW8 r;
#pragma unroll
  for (int j = 0; j < 8; ++j) r.v[j] = 0u;
  for (int j = 0; j < 32; ++j) {
    const i64 ps = pos + j;
    if (ps >= avail_lo && ps < avail_hi) r.v[j >> 2] |= (u32)in[ps] << (8 * (j & 3));
  }
  return r;
}

struct RxRange {  // words of the chunk whose windows need no edge handling
  i64 lo, hi;     // a frame [fword, fword+32K) is interior iff lo <= fword && fword+32K <= hi
  i64 len_words_full;  // words entirely below len
};
DEV RxRange rx_interior(const RxParams &p) {
  RxRange r;
  const i64 lo = p.avail_lo > p.valid_lo ? p.avail_lo : p.valid_lo;
  const i64 hi = p.avail_hi < p.valid_hi ? p.avail_hi : p.valid_hi;
  r.lo = p.aligned ? (lo + 31 >= 0 ? (lo + 31) / 32 : -((-(lo + 31) + 31) / 32)) : ((i64)1 << 62);
  r.hi = p.aligned ? (hi >= 0 ? hi / 32 : -((-hi + 31) / 32)) : -((i64)1 << 62);
  r.len_words_full = p.len / 32;
  return r;
}

template <int K> DEV void rx_fetch(const RxParams &p, const RxRange &ir, u32 lane, u32 (&x)[K][8], i64 fword) {
  const bool interior = fword >= ir.lo && fword + 32 * K <= ir.hi;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const i64 pos = (fword + (i64)(lane * K + i)) * 32;
    if (interior) {
      const uint4 *q = reinterpret_cast<const uint4 *>(p.in + pos);
      const uint4 a = __ldg(q), b = __ldg(q + 1);
      x[i][0] = a.x; x[i][1] = a.y; x[i][2] = a.z; x[i][3] = a.w;
      x[i][4] = b.x; x[i][5] = b.y; x[i][6] = b.z; x[i][7] = b.w;
    } else {
      const RxW8 r = rx_fetch_word_slow(p.in, p.avail_lo, p.avail_hi, pos);
#pragma unroll
      for (int j = 0; j < 8; ++j) x[i][j] = r.v[j];
    }
  }
}

template <int K>
DEV void rx_unpack(const RxParams &p, const RxRange &ir, Ctx<K> &c, const u32 (&x)[K][8], u32 (&pl)[8][K], i64 fword) {
  const bool interior = fword >= ir.lo && fword + 32 * K <= ir.hi;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    if (c.wb) {  // raw frame bytes for literal runs (rx_lit)
      uint4 *d = reinterpret_cast<uint4 *>(c.wb + (c.lane * K + i) * 32u);
      d[0] = make_uint4(x[i][0], x[i][1], x[i][2], x[i][3]);
      d[1] = make_uint4(x[i][4], x[i][5], x[i][6], x[i][7]);
    }
    u32 t[8];
    rx_transpose32(x[i], t);
#pragma unroll
    for (int k = 0; k < 8; ++k) pl[k][i] = t[k];
    u32 m = RX_FULL;
    if (!interior) {
      const i64 pos = (fword + (i64)(c.lane * K + i)) * 32;
      const i64 lo = p.valid_lo - pos, hi = p.valid_hi - pos;
      if (hi <= 0 || lo >= 32) m = 0u;
      else if (!(lo <= 0 && hi >= 32)) {
        const u32 a = lo <= 0 ? RX_FULL : (RX_FULL << (u32)lo);
        const u32 b = hi >= 32 ? RX_FULL : (RX_FULL >> (u32)(32 - hi));
        m = a & b;
      }
    }
    c.vm[i] = m;
  }
}

// committed mask: local words [Lw, Lw+cw), positions [0, len)
template <int K> DEV void rx_commit_mask(const RxParams &p, const RxRange &ir, Ctx<K> &c, int Lw, i64 fword) {
  const bool full = fword + Lw + (i64)c.cw <= ir.len_words_full;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const int j = (int)(c.lane * K + i);
    u32 m = (j >= Lw && j < Lw + (int)c.cw) ? RX_FULL : 0u;
    if (!full && m) {
      const i64 hi = p.len - (fword + j) * 32;
      m = hi >= 32 ? RX_FULL : (hi <= 0 ? 0u : (RX_FULL >> (u32)(32 - hi)));
    }
    c.cm[i] = m;
  }
}

DEV i64 rx_div_up(i64 a, i64 b) { return (a + b - 1) / b; }

template <class G> DEV void rx_flush(const RxParams &p, const Ctx<G::K> &c) {
  __syncwarp();
  for (int r = (int)c.lane; r < G::NR; r += 32) {
    const int gr = G::rid()[r];
    if (c.acc[3 * r]) atomicAdd(&p.counts[gr], c.acc[3 * r]);
    if (p.digests) {
      if (c.acc[3 * r + 1]) atomicAdd(&p.digests[2 * gr], c.acc[3 * r + 1]);
      if (c.acc[3 * r + 2]) atomicAdd(&p.digests[2 * gr + 1], c.acc[3 * r + 2]);
    }
  }
}

template <class G> DEV void rx_ctx_init(const RxParams &p, Ctx<G::K> &c, u64 *acc, unsigned char *lb) {
  c.lane = rx_lane();
  c.acc = acc;
  c.dense = p.dense;
  c.pitch = p.pitch;
  c.gofs = p.gofs;
  c.sign = 1ull;
  c.want_digest = p.digests != nullptr;
  c.want_dense = p.dense != nullptr;
  c.rid = G::rid();
  c.status = p.status;
  c.mlist = p.matches;
  c.mcap = p.match_cap;
  c.mtotal = p.match_total;
  c.fold = nullptr;
  c.wb = G::LIT ? lb : nullptr;
  c.ob = G::LIT ? reinterpret_cast<u32 *>(lb + 1024 * G::K) : nullptr;
  for (int r = (int)c.lane; r < 3 * G::NR; r += 32) acc[r] = 0ull;
  __syncwarp();
}

// Per-warp state scratch in shared memory (warp-private; every lane reads
// and writes the same uniform words): the body reads st[] (state carried in
// from the previous window) and accumulates nst[] (state for the next one).
DEV void rx_state_zero(u32 *a, int n, u32 lane) {
  for (int s = (int)lane; s < n; s += 32) a[s] = 0u;
  __syncwarp();
}
DEV void rx_state_copy(u32 *d, const u32 *s, int n, u32 lane) {
  for (int i = (int)lane; i < n; i += 32) d[i] = s[i];
  __syncwarp();
}
DEV bool rx_state_eq(const u32 *a, const u32 *b, int n, u32 lane) {
  bool e = true;
  for (int s = (int)lane; s < n; s += 32) e = e && (a[s] == b[s]);
  return __all_sync(RX_FULL, e);
}

// ---------------------------------------------------------------------------
// TMA (bulk async copy) staging of window bytes: one elected lane copies the
// next window's 1024*K contiguous bytes global -> shared memory, completion
// tracked by an mbarrier (transaction bytes); double-buffered per warp.
// ---------------------------------------------------------------------------
DEV u32 rx_smem_addr(const void *p) { return (u32)__cvta_generic_to_shared(p); }
DEV void rx_mbar_init(u64 *bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(rx_smem_addr(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
DEV void rx_bulk_load(void *dst, const void *src, u32 bytes, u64 *bar) {
  // the warp's generic-proxy reads of dst (ordered by the caller's
  // __syncwarp) must precede the async-proxy write
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(rx_smem_addr(bar)), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   rx_smem_addr(dst)),
               "l"(src), "r"(bytes), "r"(rx_smem_addr(bar))
               : "memory");
}
DEV void rx_mbar_wait(u64 *bar, u32 phase) {
  u32 done = 0;
  while (!done) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(rx_smem_addr(bar)), "r"(phase)
        : "memory");
  }
}

// Runs one group (traits G) over one segment (pass 1).  Windows of groups
// with K <= 2 are staged through shared memory by TMA bulk copies issued
// one window ahead; wider groups prefetch into registers.
template <class G> DEV void rx_run_segment_pf(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *lb);
template <class G>
DEV void rx_run_segment_pf_staged(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bar,
                                  unsigned char *lb);
template <class G>
DEV void rx_run_segment_cm(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bar,
                           unsigned char *lb);

template <class G>
DEV void rx_run_segment(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bars,
                        unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS;
  constexpr u32 WB = 1024u * K;  // window bytes
  if constexpr (G::PF) {
    (void)WB;
    if (K <= 4 && !p.lockstep && !p.dbg && p.cmajor && G::NC > 0)
      rx_run_segment_cm<G>(p, seg, acc, sst, tbuf, bars, lb);
    else if (K <= 4 && !p.lockstep && !p.dbg) rx_run_segment_pf_staged<G>(p, seg, acc, sst, tbuf, bars, lb);
    else rx_run_segment_pf<G>(p, seg, acc, sst, lb);
    return;
  }
  if constexpr (K <= 2) {
    const i64 len_words = rx_div_up(p.len, 32);
    const i64 nwin = rx_div_up(len_words, Bw);
    const i64 w_begin = (i64)seg * p.sw;
    const bool live = w_begin < nwin || seg == 0;
    const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
    Ctx<K> c;
    rx_ctx_init<G>(p, c, acc, lb);
    u32 pl[8][K];
    u32 xr[K][8];
    u32 *st = sst, *nst = sst + G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
    if (c.lane == 0) {
      rx_mbar_init(&bars[0], 1);
      rx_mbar_init(&bars[1], 1);
    }
    __syncwarp();
    const RxRange ir = rx_interior(p);
    const bool lockstep = p.lockstep != 0;
    bool issued0 = false, issued1 = false;
    u32 ph0 = 0, ph1 = 0;
    if (w_begin < w_end) {
      const i64 f0 = w_begin * Bw - Lw;
      if (f0 >= ir.lo && f0 + 32 * K <= ir.hi) {
        if (c.lane == 0) rx_bulk_load(tbuf, p.in + f0 * 32, WB, &bars[0]);
        issued0 = true;
      }
    }
    for (int i = 0; i < p.sw; ++i) {
      const i64 w = w_begin + i;
      const int b = i & 1;
      if (w < w_end) {
        const i64 cstart = w * Bw;
        const i64 fword = cstart - Lw;
        c.cw = (u32)((len_words - cstart) < Bw ? (len_words - cstart) : Bw);
        c.word0 = fword;
        const bool staged = b ? issued1 : issued0;
        if (staged) {
          rx_mbar_wait(&bars[b], b ? ph1 : ph0);
          if (b) { ph1 ^= 1u; issued1 = false; } else { ph0 ^= 1u; issued0 = false; }
          const uint4 *q = reinterpret_cast<const uint4 *>(tbuf + b * WB + c.lane * (32u * K));
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const uint4 a0 = q[2 * k], a1 = q[2 * k + 1];
            xr[k][0] = a0.x; xr[k][1] = a0.y; xr[k][2] = a0.z; xr[k][3] = a0.w;
            xr[k][4] = a1.x; xr[k][5] = a1.y; xr[k][6] = a1.z; xr[k][7] = a1.w;
          }
        } else {
          rx_fetch<K>(p, ir, c.lane, xr, fword);
        }
        // stage the next window into the other buffer (read by every lane
        // one window ago, released by the barrier that ended it)
        if (w + 1 < w_end) {
          const i64 nf = fword + Bw;
          if (nf >= ir.lo && nf + 32 * K <= ir.hi) {
            __syncwarp();
            if (c.lane == 0) rx_bulk_load(tbuf + (b ^ 1) * WB, p.in + nf * 32, WB, &bars[b ^ 1]);
            if (b) issued0 = true; else issued1 = true;
          }
        }
        rx_unpack<K>(p, ir, c, xr, pl, fword);
        rx_commit_mask(p, ir, c, Lw, fword);
        if (NS > 0) rx_state_zero(nst, NS, c.lane);
        G::body(c, pl, st, nst, ~0u);
        u32 *t = st;
        st = nst;
        nst = t;
        __syncwarp();
      }
      if (lockstep) __syncthreads();
    }
    if (!live) return;
    if (NS > 0) {
      u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
      for (int s = (int)c.lane; s < NS; s += 32) dst[s] = st[s];
      if (p.st_out && w_end == nwin)
        for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
    }
    rx_flush<G>(p, c);
    return;
  }
  (void)tbuf;
  (void)bars;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + G::NSMAX;
  for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
  __syncwarp();
  const RxRange ir = rx_interior(p);
  if (w_begin < w_end) rx_fetch<K>(p, ir, c.lane, xr, w_begin * Bw - Lw);
  // All warps of the CTA run this group; they step through their windows in
  // lockstep (one barrier per window) so that the SM fetches each line of
  // the group's straight-line program once for all of them.
  for (int i = 0; i < p.sw; ++i) {
    const i64 w = w_begin + i;
    if (w < w_end) {
      const i64 cstart = w * Bw;
      const i64 fword = cstart - Lw;
      c.cw = (u32)((len_words - cstart) < Bw ? (len_words - cstart) : Bw);
      c.word0 = fword;
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      if (w + 1 < w_end) rx_fetch<K>(p, ir, c.lane, xr, fword + Bw);  // prefetch the next window
      rx_commit_mask(p, ir, c, Lw, fword);
      if (NS > 0) rx_state_zero(nst, NS, c.lane);
      G::body(c, pl, st, nst, ~0u);
      u32 *t = st;
      st = nst;
      nst = t;
      __syncwarp();
    }
    if (p.lockstep) __syncthreads();
  }
  if (!live) return;
  if (NS > 0) {
    u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) dst[s] = st[s];
    if (p.st_out && w_end == nwin)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
  }
  rx_flush<G>(p, c);
}

// Fix-up / rematch (one warp per group): walk the windows in order carrying
// the true state; wherever it differs from the state pass 1 used, re-run the
// window with both states and apply (new - old) until they agree.
template <class G>
DEV void rx_fixup_group(const RxParams &p, u64 *acc, u32 *sst, unsigned char *lb, int fseg) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS, M = G::NSMAX;
  if (NS == 0) return;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 nseg = rx_div_up(nwin, p.sw);
  if (p.fix_phase == 1 && (fseg <= 0 || fseg >= nseg)) return;
  auto sstate = [&](const u32 *base, i64 seg) { return base + (seg * G::NG + G::GID) * G::NSMAX; };
  Ctx<K> c;
  rx_ctx_init<G>(p, c, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *tru = sst, *old = sst + M, *t1 = sst + 2 * M, *t2 = sst + 3 * M;
  u32 fold[G::NR * K];
  c.fold = p.match_total ? fold : nullptr;
  // re-run windows [w0, w1) with both states (old: the state the applied
  // results assumed, subtracted; tru: the true state, added) until the two
  // runs' states agree; returns whether they did
  auto walk = [&](i64 w0, i64 w1) -> bool {
    bool conv = rx_state_eq(tru, old, NS, c.lane);
    for (i64 w = w0; w < w1 && !conv; ++w) {
      const i64 cstart = w * Bw;
      const i64 fword = cstart - Lw;
      c.cw = (u32)((len_words - cstart) < Bw ? (len_words - cstart) : Bw);
      c.word0 = fword;
      const RxRange ir = rx_interior(p);
      rx_fetch<K>(p, ir, c.lane, xr, fword);
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      rx_commit_mask(p, ir, c, Lw, fword);
      // old run: subtract
      c.sign = ~0ull;
      c.want_dense = false;
      if (c.fold)
        for (int j = 0; j < G::NR * K; ++j) fold[j] = 0u;
      rx_state_zero(t1, NS, c.lane);
      G::body(c, pl, old, t1, ~0u);
      // new run: add, rewrite dense words
      c.sign = 1ull;
      c.want_dense = p.dense != nullptr;
      rx_state_zero(t2, NS, c.lane);
      G::body(c, pl, tru, t2, ~0u);
      __syncwarp();
      rx_state_copy(old, t1, NS, c.lane);
      rx_state_copy(tru, t2, NS, c.lane);
      conv = rx_state_eq(tru, old, NS, c.lane);
    }
    return conv;
  };
  if (p.mode == 1 && p.fix_phase == 1) {
    // phase 1 (one warp per (group, segment), all in parallel): pass 1 ran
    // segment fseg from a zero state; its true incoming state is taken to be
    // pass 1's end state of segment fseg-1 -- right unless that segment
    // itself did not converge here, which is flagged (seg_nc) for phase 2
    const u32 *src = sstate(p.seg_state, fseg - 1);
    for (int s = (int)c.lane; s < NS; s += 32) {
      tru[s] = src[s];
      old[s] = 0u;
    }
    __syncwarp();
    if (rx_state_eq(tru, old, NS, c.lane)) return;
    const i64 w_begin = fseg * p.sw;
    const i64 w_end = w_begin + p.sw < nwin ? w_begin + p.sw : nwin;
    if (!walk(w_begin, w_end)) {
      u32 *dst = p.seg_fix + (fseg * G::NG + G::GID) * G::NSMAX;
      for (int s = (int)c.lane; s < NS; s += 32) dst[s] = tru[s];
      if (c.lane == 0) p.seg_nc[fseg * G::NG + G::GID] = 1u;
    }
    rx_flush<G>(p, c);
    return;
  }
  if (p.mode == 1 && p.fix_phase == 2) {
    // phase 2 (one warp per group, serial over segments): only groups with a
    // segment that did not converge in phase 1.  The results applied so far
    // for segment s assume incoming A(s) = pass 1's end of s-1 (st_in for
    // s = 0); walk from the true state T where T != A(s).
    bool any = false;
    for (i64 i = c.lane; i < nseg; i += 32) any = any || p.seg_nc[i * G::NG + G::GID] != 0u;
    if (!__any_sync(RX_FULL, any)) return;
    for (int s = (int)c.lane; s < NS; s += 32) tru[s] = p.st_in ? p.st_in[G::SBASE + s] : 0u;
    __syncwarp();
    for (i64 seg = 0; seg < nseg; ++seg) {
      const u32 *a = seg == 0 ? nullptr : sstate(p.seg_state, seg - 1);
      for (int s = (int)c.lane; s < NS; s += 32) old[s] = a ? a[s] : (p.st_in ? p.st_in[G::SBASE + s] : 0u);
      __syncwarp();
      const i64 w_begin = seg * p.sw;
      const i64 w_end = w_begin + p.sw < nwin ? w_begin + p.sw : nwin;
      if (walk(w_begin, w_end)) {
        // converged: the applied run's end state stands
        const bool nc = p.seg_nc[seg * G::NG + G::GID] != 0u;
        const u32 *e = nc ? sstate(p.seg_fix, seg) : sstate(p.seg_state, seg);
        for (int s = (int)c.lane; s < NS; s += 32) tru[s] = e[s];
        __syncwarp();
      }
    }
    if (p.st_out)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = tru[s];
    rx_flush<G>(p, c);
    return;
  }
  // serial form (rematch, mode 2; and mode 1 with fix_phase 0): one warp
  // walks the segments in order carrying the true state
  for (int s = (int)c.lane; s < NS; s += 32) {
    tru[s] = p.st_in ? p.st_in[G::SBASE + s] : 0u;
    old[s] = (p.mode == 2 && p.st_assumed) ? p.st_assumed[G::SBASE + s] : 0u;
  }
  __syncwarp();
  for (i64 seg = 0; seg < nseg; ++seg) {
    const i64 w_begin = seg * p.sw;
    const i64 w_end = w_begin + p.sw < nwin ? w_begin + p.sw : nwin;
    if (p.mode == 1) {
      // the state pass 1 assumed for this segment
      for (int s = (int)c.lane; s < NS; s += 32) old[s] = seg == 0 ? (p.st_in ? p.st_in[G::SBASE + s] : 0u) : 0u;
      __syncwarp();
    }
    const bool conv = walk(w_begin, w_end);
    if (conv) {
      if (p.mode == 2) break;  // identical to the caller's run from here on
      // from here on pass 1's result stands: take its segment end state
      const u32 *src = sstate(p.seg_state, seg);
      for (int s = (int)c.lane; s < NS; s += 32) tru[s] = src[s];
      __syncwarp();
    }
    if (seg == nseg - 1 && p.st_out && (p.mode == 1 || !conv))
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = tru[s];
  }
  rx_flush<G>(p, c);
}

// ---------------------------------------------------------------------------
// Cross-regex prefilter.
// One streaming pass over the input: for every position q the 4 bytes ending
// at q form x (little-endian, byte q on top); its last two bytes index a
// 65,536-bit bigram bitmap held in shared memory; on a hit the (few) factor
// grams ending in that bigram are verified exactly against x.  A tile of 32
// blocks of 1 KiB is owned by one CTA, which records per block the factor
// ids found (deduplicated, up to 15) and per group a 32-bit word with one bit
// per block in which one of the group's factors occurs.
// ---------------------------------------------------------------------------
#define RX_PF_BLK 1024
#define RX_PF_TILE 32768

DEV u32 rx_load_u32_slow(const RxParams &p, i64 pos) {
  u32 v = 0u;
  for (int j = 0; j < 4; ++j) {
    const i64 ps = pos + j;
    if (ps >= p.avail_lo && ps < p.avail_hi) v |= (u32)p.in[ps] << (8 * j);
  }
  return v;
}

// x of position base + r (0 <= r < 20; 4 bytes ending there) from the words w0 (bytes base-4..base-1) .. w5 (base+16..base+19)
DEV u32 rx_pf_x(u32 w0, u32 w1, u32 w2, u32 w3, u32 w4, u32 w5, int r) {
  const int m = r >> 2, s = r & 3;
  const u32 lo = m == 0 ? w0 : (m == 1 ? w1 : (m == 2 ? w2 : (m == 3 ? w3 : w4)));
  const u32 hi = m == 0 ? w1 : (m == 1 ? w2 : (m == 2 ? w3 : (m == 3 ? w4 : w5)));
  return s == 3 ? hi : __funnelshift_r(lo, hi, 8 * (s + 1));
}

// One queued hit of an index bigram: its end position (offset in the tile),
// the 4 bytes ending there (xa) and the 4 bytes after them (xc); the gram
// ends d = 0..3 bytes later and is x(d) = funnel(xa, xc, 8d).  It is recorded
// in the block of the bigram's end (inside the gram, hence inside every
// window frame that contains the gram): the (group, member mask) pairs of the
// factor are ORed into the tile's shared per-(group, block) member masks.
DEV void rx_pf_record(const RxParams &p, const u32 *T, u32 *sm, u32 fid, int b) {
  const u32 f1 = T[p.pf_o_fgoff + fid + 1];
  for (u32 j = T[p.pf_o_fgoff + fid]; j < f1; ++j) {
    u32 *a = &sm[T[p.pf_o_fgent + 2 * j] * 32u + (u32)b];
    const u32 m = T[p.pf_o_fgent + 2 * j + 1];
    if ((*(volatile u32 *)a & m) != m) atomicOr(a, m);
  }
}

DEV void rx_pf_hit(const RxParams &p, const u32 *T, u32 *sm, u32 off, u32 xa, u32 xc, i64 tile_lo) {
  const u32 bg = xa >> 16, wi = bg >> 5, bit = bg & 31u;
  const u32 idx = T[2048 + wi] + __popc(T[wi] & ((1u << bit) - 1u));
  u32 shapes = T[4096 + idx];
  const int b = (int)(off >> 10);
  const i64 q0 = tile_lo + off;
  const u32 hmask = (1u << p.pf_hbits) - 1u;
  const u32 *H = T + p.pf_o_ent;
  while (shapes) {
    const u32 sh = __ffs(shapes) - 1;
    shapes &= shapes - 1u;
    const u32 k = sh / 3u + 2u, d = sh - 3u * (k - 2u);
    const u32 mask = k == 4u ? 0xffffffffu : (0xffffffffu << (8u * (4u - k)));
    const u32 key = (d == 0u ? xa : __funnelshift_r(xa, xc, 8u * d)) & mask;
    const i64 q = q0 + d;
    if (q >= p.avail_hi || q - (i64)k + 1 < p.avail_lo) continue;
    u32 h = ((key ^ (sh * 0x85EBCA6Bu)) * 0x9E3779B1u) >> (32u - p.pf_hbits);
    for (;;) {
      const u32 tag = H[2 * h + 1];
      if (tag == 0u) break;
      if (H[2 * h] == key && ((tag >> 1) & 127u) == sh) rx_pf_record(p, T, sm, tag >> 8, b);
      h = (h + 1u) & hmask;
    }
  }
}

// smem: [tables (if they fit) | member masks NG x 32 | per-warp hit queues 32 x 3]
DEV void rx_prefilter_run(const RxParams &p, int NG, bool tab_in_smem) {
  extern __shared__ __align__(16) u32 pf_smem[];
  const int tid = threadIdx.x, nt = blockDim.x;
  const u32 tw = tab_in_smem ? ((p.pf_words + 3u) & ~3u) : 4096u;
  u32 *tab = pf_smem;
  for (u32 i = tid; i < tw && i < p.pf_words; i += nt) tab[i] = __ldg(&p.pf_tab[i]);
  // l1 + rank are always staged; the rest is read through T
  const u32 *T = tab_in_smem ? (const u32 *)tab : p.pf_tab;
  u32 *sm = pf_smem + tw;                     // [NG][32 blocks] member masks
  u32 *wq = sm + 32 * NG + 96 * (tid >> 5);  // per-warp hit queue: 32 x {off, xa, xc}
  const u32 lane = rx_lane();
  const i64 span = p.avail_hi - p.avail_lo;
  const i64 ntiles = (span + RX_PF_TILE - 1) / RX_PF_TILE;
  for (i64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
    for (int i = tid; i < 32 * NG; i += nt) sm[i] = 0u;
    __syncthreads();
    const i64 tile_lo = p.avail_lo + t * RX_PF_TILE;
    for (int j = 0; j < RX_PF_TILE / 16; j += nt) {
      const i64 base = tile_lo + (i64)(j + tid) * 16;
      u32 w1, w2, w3, w4;
      if (p.pf_aligned && base + 16 <= p.avail_hi) {
        const uint4 v = __ldg(reinterpret_cast<const uint4 *>(p.in + base));
        w1 = v.x; w2 = v.y; w3 = v.z; w4 = v.w;
      } else {
        w1 = rx_load_u32_slow(p, base);
        w2 = rx_load_u32_slow(p, base + 4);
        w3 = rx_load_u32_slow(p, base + 8);
        w4 = rx_load_u32_slow(p, base + 12);
      }
      u32 w0 = __shfl_up_sync(RX_FULL, w4, 1);
      if (lane == 0) w0 = rx_load_u32_slow(p, base - 4);
      u32 w5 = __shfl_down_sync(RX_FULL, w1, 1);
      if (lane == 31) w5 = rx_load_u32_slow(p, base + 16);
      // pass 1: bigram bitmap test of the 16 positions -> hit mask
      u32 hm = 0u;
#pragma unroll
      for (int r = 0; r < 16; ++r) {
        const u32 x = rx_pf_x(w0, w1, w2, w3, w4, w5, r);
        const u32 bg = x >> 16;
        hm |= ((tab[bg >> 5] >> (bg & 31)) & 1u) << r;
      }
      const i64 rem = p.avail_hi - base;
      if (rem < 16) hm &= rem <= 0 ? 0u : ((1u << rem) - 1u);
      // pass 2: the warp's hits are compacted into a queue of 32 and checked
      // one per lane (exact gram compare)
      u32 qn = 0;
      for (;;) {
        const u32 bal = __ballot_sync(RX_FULL, hm != 0u);
        if (bal) {
          const u32 rk = __popc(bal & ((1u << lane) - 1u));
          if (hm != 0u && qn + rk < 32u) {
            const int r = __ffs(hm) - 1;
            hm &= hm - 1u;
            u32 *e = wq + 3 * (qn + rk);
            e[0] = (u32)(base + r - tile_lo);
            e[1] = rx_pf_x(w0, w1, w2, w3, w4, w5, r);
            e[2] = rx_pf_x(w0, w1, w2, w3, w4, w5, r + 4);
          }
          qn = qn + __popc(bal) < 32u ? qn + __popc(bal) : 32u;
        }
        if (qn == 32u || (bal == 0u && qn > 0u)) {
          __syncwarp();
          if (lane < qn) rx_pf_hit(p, T, sm, wq[3 * lane], wq[3 * lane + 1], wq[3 * lane + 2], tile_lo);
          __syncwarp();
          qn = 0;
        }
        if (bal == 0u) break;
      }
    }
    __syncthreads();
    // one warp per group: lane b holds block b's member mask; the group's
    // tile word of block bits is their ballot
    const i64 nblk = 32 * p.pf_ntiles;
    for (int g = tid >> 5; g < NG; g += nt >> 5) {
      const u32 v = sm[32 * g + lane];
      const u32 bal = __ballot_sync(RX_FULL, v != 0u);
      if (lane == 0) p.pf_gbits[(i64)g * p.pf_ntiles + t] = bal;
      if (v) p.pf_mmask[(i64)g * nblk + t * 32 + lane] = v;
    }
    __syncthreads();
  }
}

// first block >= b0 (and <= bmax) whose bit is set in the group's bitmap;
// returns bmax + 1 if none (warp-uniform)
DEV i64 rx_pf_next(const u32 *gb, i64 b0, i64 bmax, u32 lane) {
  for (i64 w0 = b0 >> 5; w0 <= (bmax >> 5); w0 += 32) {
    const i64 wi = w0 + lane;
    u32 v = wi <= (bmax >> 5) ? gb[wi] : 0u;
    if (wi == (b0 >> 5)) v &= RX_FULL << (b0 & 31);
    const u32 bal = __ballot_sync(RX_FULL, v != 0u);
    if (bal) {
      const int l = __ffs(bal) - 1;
      const u32 vv = __shfl_sync(RX_FULL, v, l);
      const i64 b = (w0 + l) * 32 + (__ffs(vv) - 1);
      return b <= bmax ? b : bmax + 1;
    }
  }
  return bmax + 1;
}

DEV i64 rx_floor_div(i64 a, i64 b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }

// Pass 1 with the prefilter: windows whose frame holds no factor of the group
// and into which no state flows are skipped without loading a byte; the
// others run only the members whose factor occurs in the frame, that carry
// state, or that have no factor (G::ALWAYS).
template <class G> DEV void rx_run_segment_pf(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + G::NSMAX;
  for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
  __syncwarp();
  const RxRange ir = rx_interior(p);
  const u32 *gb = p.pf_gbits + (i64)G::GID * p.pf_ntiles;
  auto frame_blocks = [&](i64 w, i64 &b0, i64 &b1) {
    i64 flo = (w * Bw - Lw) * 32, fhi = flo + 1024 * K;
    if (flo < p.avail_lo) flo = p.avail_lo;
    if (fhi > p.avail_hi) fhi = p.avail_hi;
    if (fhi <= flo) fhi = flo + 1;
    b0 = (flo - p.avail_lo) >> 10;
    b1 = (fhi - 1 - p.avail_lo) >> 10;
  };
  i64 bmax = 0;
  if (w_begin < w_end) {
    i64 t0;
    frame_blocks(w_end - 1, t0, bmax);
  }
  // lockstep (p.lockstep): the CTA's warps step through window i together
  // (one barrier per step) so that they fetch the group's code together;
  // otherwise each warp jumps to its next window with a factor hit
  const bool lockstep = p.lockstep != 0;
  i64 w = w_begin;
  int step = 0;
  while (lockstep ? step < p.sw : w < w_end) {
    if (lockstep) {
      if (step > 0) __syncthreads();
      w = w_begin + step;
      ++step;
      if (w >= w_end) continue;
    }
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    bool pend = false;
    if (NS > 0) {
      bool any = false;
      for (int s = (int)c.lane; s < NS; s += 32) any = any || st[s] != 0u;
      pend = __any_sync(RX_FULL, any);
    }
    if (p.stats && c.lane == 0) atomicAdd(&p.stats[3], 1ull);  // [3] window visits (checks)
    if (p.dbg == 1) {
      if (lockstep) continue;
      ++w;
      continue;
    }
    if (!pend && G::ALWAYS == 0u) {
      const i64 b = rx_pf_next(gb, b0, lockstep ? b1 : bmax, c.lane);
      if (lockstep && b > b1) continue;
      if (b > b1) {
        if (b > bmax) break;
        // the first window whose frame reaches block b
        const i64 pos = p.avail_lo + b * RX_PF_BLK;
        const i64 wn = rx_floor_div(rx_floor_div(pos, 32) + Lw - 32 * K, Bw) + 1;
        w = wn > w + 1 ? wn : w + 1;
        continue;
      }
    }
    // members whose factor occurs in one of the frame's blocks (lane i
    // looks at block b0 + i; a frame spans a few blocks)
    const u32 *mm = p.pf_mmask + (i64)G::GID * 32 * p.pf_ntiles;
    u32 mine = 0u;
    for (i64 b = b0 + c.lane; b <= b1; b += 32)
      if ((gb[b >> 5] >> (b & 31)) & 1u) mine |= mm[b];
    const u32 rmask = __reduce_or_sync(RX_FULL, mine);
    if (p.stats && c.lane == 0) {
      // [0] active windows [1] of them only for carried state [2] members hit
      atomicAdd(&p.stats[0], 1ull);
      if (rmask == 0u) atomicAdd(&p.stats[1], 1ull);
      atomicAdd(&p.stats[2], (u64)__popc(rmask));
    }
    const i64 cstart = w * Bw;
    const i64 fword = cstart - Lw;
    c.cw = (u32)((len_words - cstart) < Bw ? (len_words - cstart) : Bw);
    c.word0 = fword;
    rx_fetch<K>(p, ir, c.lane, xr, fword);
    rx_unpack<K>(p, ir, c, xr, pl, fword);
    rx_commit_mask(p, ir, c, Lw, fword);
    if (NS > 0) rx_state_zero(nst, NS, c.lane);
    if (p.dbg == 2) {
      if (c.lane == 0 && (pl[0][0] ^ pl[7][K - 1]) == 0x12345u) atomicAdd(p.status, 0u);  // keep the loads
    } else {
      G::body(c, pl, st, nst, rmask);
    }
    u32 *t = st;
    st = nst;
    nst = t;
    __syncwarp();
    if (!lockstep) ++w;
  }
  if (lockstep && step > 0) __syncthreads();
  if (!live) return;
  if (NS > 0) {
    u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) dst[s] = st[s];
    if (p.st_out && w_end == nwin)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
  }
  rx_flush<G>(p, c);
}

// Sparse pass 1 with a one-window lookahead (the default): while the body
// of window w runs, the bytes of the window expected next -- w + 1 if state
// flows into w (it usually flows on), else the next window whose frame holds
// a factor of the group -- are already on their way into a per-warp shared
// buffer by a TMA bulk copy.  A wrong guess costs a synchronous global load;
// the window order and the set of windows run are exactly those of
// rx_run_segment_pf (running an extra window with no state and no factor is
// harmless: its output and state are zero).
template <class G>
DEV void rx_run_segment_pf_staged(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bar,
                                  unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS;
  constexpr u32 WB = 1024u * K;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + G::NSMAX;
  for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
  if (c.lane == 0) rx_mbar_init(bar, 1);
  __syncwarp();
  const RxRange ir = rx_interior(p);
  const u32 *gb = p.pf_gbits + (i64)G::GID * p.pf_ntiles;
  const u32 *mm = p.pf_mmask + (i64)G::GID * 32 * p.pf_ntiles;
  auto frame_blocks = [&](i64 w, i64 &b0, i64 &b1) {
    i64 flo = (w * Bw - Lw) * 32, fhi = flo + 1024 * K;
    if (flo < p.avail_lo) flo = p.avail_lo;
    if (fhi > p.avail_hi) fhi = p.avail_hi;
    if (fhi <= flo) fhi = flo + 1;
    b0 = (flo - p.avail_lo) >> 10;
    b1 = (fhi - 1 - p.avail_lo) >> 10;
  };
  i64 bmax = 0;
  if (w_begin < w_end) {
    i64 t0;
    frame_blocks(w_end - 1, t0, bmax);
  }
  auto pending = [&](const u32 *a) -> bool {
    if (NS == 0) return false;
    bool any = false;
    for (int s = (int)c.lane; s < NS; s += 32) any = any || a[s] != 0u;
    return __any_sync(RX_FULL, any);
  };
  // first window >= w whose frame holds a factor of the group (w_end if none)
  auto next_hit = [&](i64 w) -> i64 {
    if (w >= w_end) return w_end;
    if (G::ALWAYS != 0u) return w;
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    const i64 b = rx_pf_next(gb, b0, bmax, c.lane);
    if (b > bmax) return w_end;
    if (b <= b1) return w;
    const i64 pos = p.avail_lo + b * RX_PF_BLK;
    const i64 wn = rx_floor_div(rx_floor_div(pos, 32) + Lw - 32 * K, Bw) + 1;
    const i64 r = wn > w + 1 ? wn : w + 1;
    return r < w_end ? r : w_end;
  };
  i64 staged = -1;  // window whose bytes are in flight / in tbuf (-1: none)
  u32 phase = 0;
  auto stage = [&](i64 w) {
    const i64 f = w * Bw - Lw;
    if (w < w_end && f >= ir.lo && f + 32 * K <= ir.hi) {
      __syncwarp();
      if (c.lane == 0) rx_bulk_load(tbuf, p.in + f * 32, WB, bar);
      staged = w;
    }
  };
  auto retire = [&]() {  // wait for the copy in flight (keeps the mbarrier phase in step)
    rx_mbar_wait(bar, phase);
    phase ^= 1u;
    staged = -1;
  };
  i64 w = pending(st) ? w_begin : next_hit(w_begin);
  if (w < w_end) stage(w);
  while (w < w_end) {
    const bool pend_in = pending(st);
    if (p.stats && c.lane == 0) atomicAdd(&p.stats[3], 1ull);
    const i64 fword = w * Bw - Lw;
    if (staged == w) {
      retire();
      const uint4 *q = reinterpret_cast<const uint4 *>(tbuf + c.lane * (32u * K));
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const uint4 a0 = q[2 * k], a1 = q[2 * k + 1];
        xr[k][0] = a0.x; xr[k][1] = a0.y; xr[k][2] = a0.z; xr[k][3] = a0.w;
        xr[k][4] = a1.x; xr[k][5] = a1.y; xr[k][6] = a1.z; xr[k][7] = a1.w;
      }
    } else {
      if (staged >= 0 && staged < w) retire();  // a stale guess: drain it
      rx_fetch<K>(p, ir, c.lane, xr, fword);
    }
    // guess the next window and start its copy before the body runs
    if (staged < 0) {
      const i64 guess = pend_in ? w + 1 : next_hit(w + 1);
      stage(guess);
    }
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    u32 mine = 0u;
    for (i64 b = b0 + c.lane; b <= b1; b += 32)
      if ((gb[b >> 5] >> (b & 31)) & 1u) mine |= mm[b];
    const u32 rmask = __reduce_or_sync(RX_FULL, mine);
    if (p.stats && c.lane == 0) {
      atomicAdd(&p.stats[0], 1ull);
      if (rmask == 0u) atomicAdd(&p.stats[1], 1ull);
      atomicAdd(&p.stats[2], (u64)__popc(rmask));
    }
    c.cw = (u32)((len_words - w * Bw) < Bw ? (len_words - w * Bw) : Bw);
    c.word0 = fword;
    rx_unpack<K>(p, ir, c, xr, pl, fword);
    rx_commit_mask(p, ir, c, Lw, fword);
    if (NS > 0) rx_state_zero(nst, NS, c.lane);
    G::body_i(c, pl, st, nst, rmask);
    u32 *t = st;
    st = nst;
    nst = t;
    __syncwarp();
    w = pending(st) ? w + 1 : next_hit(w + 1);
  }
  if (staged >= 0) retire();
  if (!live) return;
  if (NS > 0) {
    u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) dst[s] = st[s];
    if (p.st_out && w_end == nwin)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
  }
  rx_flush<G>(p, c);
}

// Cluster-major sparse pass 1 (the default).  The
// segment is walked once per factor cluster of the group, running only that
// cluster's out-of-line code (G::cbody) in the windows whose frame holds one
// of its factors or into which its own state flows.  A cluster's code stays
// in the SM's instruction caches across consecutive windows (one straight-
// line body per window over the whole group thrashed them: the top stall was
// "no instruction"), at the price of re-loading and re-transposing a window
// for each cluster that runs in it.  Clusters own disjoint state slots, so
// running them one after the other over the segment computes exactly what
// the window-major order computes.  With cm_sync the CTA's warps (same group,
// consecutive segments) step from cluster to cluster together.
template <class G>
DEV void rx_run_segment_cm(const RxParams &p, int seg, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bar,
                           unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw;
  constexpr u32 WB = 1024u * K;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + G::NSMAX;
  if (c.lane == 0) rx_mbar_init(bar, 1);
  __syncwarp();
  const RxRange ir = rx_interior(p);
  const u32 *gb = p.pf_gbits + (i64)G::GID * p.pf_ntiles;
  const u32 *mm = p.pf_mmask + (i64)G::GID * 32 * p.pf_ntiles;
  auto frame_blocks = [&](i64 w, i64 &b0, i64 &b1) {
    i64 flo = (w * Bw - Lw) * 32, fhi = flo + 1024 * K;
    if (flo < p.avail_lo) flo = p.avail_lo;
    if (fhi > p.avail_hi) fhi = p.avail_hi;
    if (fhi <= flo) fhi = flo + 1;
    b0 = (flo - p.avail_lo) >> 10;
    b1 = (fhi - 1 - p.avail_lo) >> 10;
  };
  i64 bmax = 0;
  if (w_begin < w_end) {
    i64 t0;
    frame_blocks(w_end - 1, t0, bmax);
  }
  // members of the group whose factor occurs in window w's frame
  auto frame_hits = [&](i64 w) -> u32 {
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    u32 mine = 0u;
    for (i64 b = b0 + c.lane; b <= b1; b += 32)
      if ((gb[b >> 5] >> (b & 31)) & 1u) mine |= mm[b];
    return __reduce_or_sync(RX_FULL, mine);
  };
  // first window >= w whose frame holds a factor of the group (w_end if none)
  auto next_group_hit = [&](i64 w) -> i64 {
    if (w >= w_end) return w_end;
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    const i64 b = rx_pf_next(gb, b0, bmax, c.lane);
    if (b > bmax) return w_end;
    if (b <= b1) return w;
    const i64 pos = p.avail_lo + b * RX_PF_BLK;
    const i64 wn = rx_floor_div(rx_floor_div(pos, 32) + Lw - 32 * K, Bw) + 1;
    const i64 r = wn > w + 1 ? wn : w + 1;
    return r < w_end ? r : w_end;
  };
  i64 staged = -1;
  u32 phase = 0;
  auto stage = [&](i64 w) {
    const i64 f = w * Bw - Lw;
    if (w < w_end && f >= ir.lo && f + 32 * K <= ir.hi) {
      __syncwarp();
      if (c.lane == 0) rx_bulk_load(tbuf, p.in + f * 32, WB, bar);
      staged = w;
    }
  };
  auto retire = [&]() {
    rx_mbar_wait(bar, phase);
    phase ^= 1u;
    staged = -1;
  };
  for (int ci = 0; ci < G::NC; ++ci) {
    const int s0 = G::cslot(ci), s1 = G::cslot(ci + 1);
    const u32 cm = G::cmask(ci);
    const bool always = G::calways(ci);
    for (int s = s0 + (int)c.lane; s < s1; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
    __syncwarp();
    auto pending = [&](const u32 *a) -> bool {
      bool any = false;
      for (int s = s0 + (int)c.lane; s < s1; s += 32) any = any || a[s] != 0u;
      return __any_sync(RX_FULL, any);
    };
    // first window >= w in which this cluster must run (no state pending)
    auto next_c = [&](i64 w) -> i64 {
      if (always) return w < w_end ? w : w_end;
      for (;;) {
        w = next_group_hit(w);
        if (w >= w_end) return w_end;
        if (frame_hits(w) & cm) return w;
        ++w;
      }
    };
    i64 w = pending(st) ? w_begin : next_c(w_begin);
    if (w < w_end) stage(w);
    while (w < w_end) {
      const bool pend_in = pending(st);
      const i64 fword = w * Bw - Lw;
      if (staged == w) {
        retire();
        const uint4 *q = reinterpret_cast<const uint4 *>(tbuf + c.lane * (32u * K));
#pragma unroll
        for (int k = 0; k < K; ++k) {
          const uint4 a0 = q[2 * k], a1 = q[2 * k + 1];
          xr[k][0] = a0.x; xr[k][1] = a0.y; xr[k][2] = a0.z; xr[k][3] = a0.w;
          xr[k][4] = a1.x; xr[k][5] = a1.y; xr[k][6] = a1.z; xr[k][7] = a1.w;
        }
      } else {
        if (staged >= 0 && staged < w) retire();
        rx_fetch<K>(p, ir, c.lane, xr, fword);
      }
      if (staged < 0) stage(pend_in ? w + 1 : next_c(w + 1));
      const u32 rmask = frame_hits(w) & cm;
      if (p.stats && c.lane == 0) {
        atomicAdd(&p.stats[0], 1ull);
        if (rmask == 0u) atomicAdd(&p.stats[1], 1ull);
        atomicAdd(&p.stats[2], (u64)__popc(rmask));
        atomicAdd(&p.stats[3], 1ull);
      }
      c.cw = (u32)((len_words - w * Bw) < Bw ? (len_words - w * Bw) : Bw);
      c.word0 = fword;
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      rx_commit_mask(p, ir, c, Lw, fword);
      for (int s = s0 + (int)c.lane; s < s1; s += 32) nst[s] = 0u;
      __syncwarp();
      G::cbody(ci, c, pl, st, nst, rmask);
      u32 *t = st;
      st = nst;
      nst = t;
      __syncwarp();
      w = pending(st) ? w + 1 : next_c(w + 1);
    }
    if (staged >= 0) retire();
    if (live && s1 > s0) {
      u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
      for (int s = s0 + (int)c.lane; s < s1; s += 32) dst[s] = st[s];
      if (p.st_out && w_end == nwin)
        for (int s = s0 + (int)c.lane; s < s1; s += 32) p.st_out[G::SBASE + s] = st[s];
    }
    __syncwarp();
    if (p.cm_sync) __syncthreads();
  }
  if (!live) return;
  rx_flush<G>(p, c);
}
