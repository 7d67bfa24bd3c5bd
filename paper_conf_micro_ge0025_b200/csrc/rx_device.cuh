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
//  * a cross-regex prefilter (rx_prefilter_run) decides which clusters of a
//    group run in which windows: mode A -- where a first factor occurs or
//    state flows in; mode B -- only where an output factor occurs, with the
//    state the window needs reconstructed by a convergence walk-back
//    (rx_walk_back);
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
// emission context: per-warp, in shared memory (the out-of-line epilogue
// reads it there instead of taking a large struct by value)
// ---------------------------------------------------------------------------
struct RxOut {
  u64 *acc;         // per-warp shared accumulators [NR][3] (count, d1, d2)
  u32 *dense;       // nullable
  u64 pitch;
  i64 gofs;         // global position of chunk position 0
  u64 sign;         // 1 (add) or 2^64-1 (subtract; fix-up pass)
  const int *rid;   // group member -> global regex id
  u32 *status;
  u64 *mlist;       // nullable: compacted match list, {regex, pos} pairs (rx_match_t)
  u64 mcap;
  u64 *mtotal;
  u32 *fold;        // fix-up only: [NR][K] output words of the "old" run (match-list delta)
  int want_digest, want_dense;
};

// window context (scalars only: the 8 basis streams live in a register array
// of the segment loop and are passed to the body separately)
template <int K>
struct Ctx {
  u32 vm[K];    // positions holding real stream bytes
  u32 cm[K];    // committed positions of this window inside [0, len)
  u32 lane;
  u32 cw;       // committed words of this window
  i64 word0;    // chunk word index of local word 0
  RxOut *o;     // shared memory
  unsigned char *wb;  // nullable (groups without literal runs): the frame's bytes, frame position f at wb[f]
  u32 *ob;            // literal-run output scratch, 32*K words (per warp)
  bool walk;          // state-only run (mode-B walk-back): no output
  bool dense;         // dense output requested (mirrors o->want_dense)
  bool fast;          // counts only (no digests, dense streams or match list) and sign +1: the
                      // generated epilogue adds the popcount to acc inline, without rx_emit
  u64 *acc;           // per-warp shared accumulators [NR][3] (== o->acc)
};

// ---------------------------------------------------------------------------
// epilogue (called only when the output has a set bit in the committed
// range, or when dense output is requested): popcount -> REDUX, digests,
// dense store, match list
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
// prefix sum.  The fix-up's "old" run (sign = -1) records its words in o->fold
// and the "new" run lists only the bits the old one lacked: match sets are
// monotone in the incoming state (every operation on state streams is AND /
// OR / Advance / add-with-carry of a marker into a class), so new covers old;
// a violation is flagged in status bit 2 instead of being silently dropped.
template <int K>
DEV void rx_emit_list(const RxOut *o, int r, u32 lane, i64 word0, const u32 (&m)[K]) {
  u32 mm[K];
  u32 cnt = 0;
  bool lost = false;
#pragma unroll
  for (int i = 0; i < K; ++i) {
    if (o->fold && o->sign == ~0ull) {
      o->fold[r * K + i] = m[i];
      mm[i] = 0u;
    } else if (o->fold) {
      lost = lost || (o->fold[r * K + i] & ~m[i]) != 0u;
      mm[i] = m[i] & ~o->fold[r * K + i];
    } else {
      mm[i] = m[i];
    }
    cnt += __popc(mm[i]);
  }
  if (lost) atomicOr(o->status, 4u);
  u32 incl = cnt;
#pragma unroll
  for (int s = 1; s < 32; s <<= 1) {
    const u32 t = __shfl_up_sync(RX_FULL, incl, s);
    if (lane >= (u32)s) incl += t;
  }
  const u32 tot = __shfl_sync(RX_FULL, incl, 31);
  if (tot == 0u) return;
  u64 base = 0;
  if (lane == 0) base = atomicAdd(o->mtotal, (u64)tot);
  base = __shfl_sync(RX_FULL, base, 0) + (incl - cnt);
  const u64 reg = (u64)(u32)o->rid[r];
#pragma unroll
  for (int i = 0; i < K; ++i) {
    u32 b = mm[i];
    const i64 wpos = o->gofs + (word0 + (i64)(lane * K + i)) * 32;
    while (b) {
      const int t = __ffs(b) - 1;
      b &= b - 1u;
      if (base < o->mcap) {
        o->mlist[2 * base] = reg;
        o->mlist[2 * base + 1] = (u64)(wpos + t);
      }
      ++base;
    }
  }
}

// m: the output words already masked to the committed positions; cwb: bit i
// set if word i of this lane is committed (dense stores)
template <int K>
__device__ __noinline__ void rx_emit(const RxOut *o, int r, u32 lane, i64 word0, const V<K> m, u32 cwb) {
  u32 any = 0u;
#pragma unroll
  for (int i = 0; i < K; ++i) any |= m.w[i];
  if (o->want_dense) {
    u32 *row = o->dense + (u64)o->rid[r] * o->pitch;
#pragma unroll
    for (int i = 0; i < K; ++i)
      if ((cwb >> i) & 1u) row[word0 + (i64)(lane * K + i)] = m.w[i];
  }
  if (!__any_sync(RX_FULL, any != 0u)) return;
  u32 cnt = 0;
#pragma unroll
  for (int i = 0; i < K; ++i) cnt += __popc(m.w[i]);
  const u32 tot = __reduce_add_sync(RX_FULL, cnt);
  u64 d1 = 0, d2 = 0;
  if (o->want_digest) {
#pragma unroll
    for (int i = 0; i < K; ++i) {
      u32 b = m.w[i];
      const i64 base = o->gofs + (word0 + (i64)(lane * K + i)) * 32;
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
  if (lane == 0) {
    o->acc[3 * r + 0] += o->sign * (u64)tot;
    o->acc[3 * r + 1] += o->sign * d1;
    o->acc[3 * r + 2] += o->sign * d2;
  }
  if (o->mtotal) {
    u32 mm[K];
#pragma unroll
    for (int i = 0; i < K; ++i) mm[i] = m.w[i];
    rx_emit_list<K>(o, r, lane, word0, mm);
  }
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
DEV u32 rx_ld_s8(u32 a) {
  u32 v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
DEV u32 rx_ld_s32(u32 a) {
  u32 v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
DEV void rx_st_s32(u32 a, u32 v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
DEV void rx_red_or_s32(u32 a, u32 v) { asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }

// wbs / obs: shared-space addresses of the frame bytes and of the per-warp
// output words (explicit ld/st/red.shared: handed to an out-of-line function
// as generic pointers they compiled to generic loads and GPU-scope generic
// atomics, profiles/r2_ncu_r2n*)
template <int K>
__device__ __noinline__ V<K> rx_lit(const u32 lane, const u32 wbs, const u32 obs, const V<K> v,
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
  for (int i = 0; i < K; ++i) rx_st_s32(obs + 4u * (lane * K + i), 0u);
  __syncwarp();
  const int F = 1024 * K;
  const u32 l0 = __ldg(lit);
#pragma unroll
  for (int i = 0; i < K; ++i) {
    u32 b = v.w[i];
    while (b) {
      const int t = __ffs(b) - 1;
      b &= b - 1u;
      const int q = (int)((lane * K + i) * 32u) + t;
      const int e = q + n;
      if (e >= F || rx_ld_s8(wbs + (u32)q + 1u) != l0) continue;
      int j = 1;
      while (j < n && rx_ld_s8(wbs + (u32)(q + 1 + j)) == (u32)__ldg(lit + j)) ++j;
      if (j == n) rx_red_or_s32(obs + 4u * (u32)(e >> 5), 1u << (e & 31));
    }
  }
  __syncwarp();
#pragma unroll
  for (int i = 0; i < K; ++i) r.w[i] = rx_ld_s32(obs + 4u * (lane * K + i));
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
  int modeb;                // mode B allowed (plain rx_match: no chunk state in/out)
  int lockstep;             // sparse pass 1 (rx_run_segment_pf): 0 free-running warps, 1 cluster lockstep
                            // (a barrier per cluster), 2 round lockstep (a barrier per window round)
  // cross-regex prefilter (rx_prefilter_run below; rx_prefilter.cpp
  // build_prefilter documents the table blob)
  const u32 *pf_tab;
  u32 pf_words, pf_smem_words;
  u32 pf_b4bits, pf_b3bits, pf_hbits;
  u32 pf_o_b3, pf_o_b2, pf_o_ht, pf_o_ext, pf_o_fgoff, pf_o_fgent;
  u32 *pf_gbits;            // [NG][ntiles]: bit b of word t = a factor of the group occurs in block 32t+b
  u32 *pf_mmask;            // [NG][32*ntiles]: members whose FIRST factor occurs in the block
  u32 *pf_omask;            // [NG][32*ntiles]: members whose OUTPUT factor occurs in the block (null: the
                            // program has no output factor, mode B off)
                            // (both written wherever a pf_gbits bit is set)
  u32 *pf_cnt;              // [NG][32][2]: blocks with a first / output factor hit per member (mode choice)
  i64 pf_ntiles;
  int pf_on;
  u64 *stats;               // nullable: counters (RX_F_STATS), see rx_run_segment_pf
  u64 *matches;             // nullable: rx_match_t[match_cap] as u64 pairs {regex, pos}
  u64 match_cap;
  u64 *match_total;         // u64: matches found (may exceed match_cap)
  int fix_phase;            // mode 1: 1 = parallel per segment, 2 = serial remainder
  u32 *seg_fix;             // [nseg_max][G][NSMAX]: phase-1 end state of a segment that did not converge
  u32 *seg_nc;              // [nseg_max][G]: that segment did not converge in phase 1
  // rx_match_batch (one launch sequence for all streams): stream s is
  // in[batch_off[s] .. batch_off[s+1]); pass-1 "segment" j = streams
  // [j*batch_spw, (j+1)*batch_spw), whose warp runs each whole with its own
  // copy of these parameters (rx_batch_view)
  const u64 *batch_off;     // device u64[batch_n + 1] (null: not a batch)
  i64 batch_n;
  i64 batch_spw;            // streams per pass-1 segment (one warp runs them one after the other)
  i64 pf_shift;             // prefilter block coordinates = stream position + pf_shift
};

// CTA header of the dynamic shared memory (pass 1 and fix-up): the launch
// parameters (copied once per CTA by the kernel, then read with LDS at fixed
// offsets) and the cluster-lockstep union words; the per-warp areas follow.
#define RX_CTA_HDR 512
static_assert(sizeof(RxParams) <= 496, "RxParams must fit the CTA header");
DEV unsigned char *rx_dyn_smem() {
  extern __shared__ __align__(16) u64 rx_smem[];
  return reinterpret_cast<unsigned char *>(rx_smem);
}
DEV const RxParams &rx_cta_params() { return *reinterpret_cast<const RxParams *>(rx_dyn_smem()); }
DEV u32 *rx_cta_union() { return reinterpret_cast<u32 *>(rx_dyn_smem() + 496); }
DEV unsigned char *rx_warp_smem(int warp, int per) { return rx_dyn_smem() + RX_CTA_HDR + (size_t)warp * per; }
DEV void rx_cta_params_store(const RxParams &p) {
  const u32 *src = reinterpret_cast<const u32 *>(&p);
  u32 *dst = reinterpret_cast<u32 *>(rx_dyn_smem());
  for (int i = threadIdx.x; i < (int)(sizeof(RxParams) / 4); i += blockDim.x) dst[i] = src[i];
  __syncthreads();
}

// rx_match_batch: this warp's stream s as a whole input of its own (zero
// state in, nothing readable outside it), written over a per-warp copy of the
// launch parameters; warps beyond the last stream get an empty stream (they
// still take part in the CTA's lockstep barriers)
DEV const RxParams &rx_batch_view(const RxParams &pc, RxParams *wp, i64 s, int nreg) {
  const u32 lane = threadIdx.x & 31u;
  const u32 *src = reinterpret_cast<const u32 *>(&pc);
  u32 *dst = reinterpret_cast<u32 *>(wp);
  for (int i = (int)lane; i < (int)(sizeof(RxParams) / 4); i += 32) dst[i] = src[i];
  __syncwarp();
  if (lane == 0) {
    const bool ok = s < pc.batch_n;
    const u64 o0 = ok ? pc.batch_off[s] : 0ull, o1 = ok ? pc.batch_off[s + 1] : 0ull;
    const i64 len = (i64)(o1 - o0);
    wp->in = pc.in + o0;
    wp->avail_lo = wp->valid_lo = 0;
    wp->avail_hi = wp->valid_hi = wp->len = len;
    wp->gofs = pc.gofs + (i64)o0;
    wp->pf_shift = (i64)o0;
    const i64 ss = ok ? s : 0;
    wp->counts = pc.counts + ss * nreg;
    wp->digests = pc.digests ? pc.digests + 2 * ss * nreg : nullptr;
    wp->dense = pc.dense ? pc.dense + (u64)ss * nreg * pc.pitch : nullptr;
    wp->aligned = ((reinterpret_cast<unsigned long long>(wp->in) & 15ull) == 0ull) ? 1 : 0;
    wp->nseg_max = 1;  // sw: the host's window count of the longest stream
    wp->seg_state = nullptr;
    wp->st_in = nullptr;
    wp->st_out = nullptr;
    wp->modeb = 0;
  }
  __syncwarp();
  return *wp;
}

// split prologue (software pipelining): rx_fetch issues the 128-bit loads of
// a window into registers, rx_unpack transposes them.  Interior windows (all
// bytes readable and valid, 16-byte aligned) take the straight path; edge
// windows go through an out-of-line byte loader.
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
  const u64 *acc = c.o->acc;
  for (int r = (int)c.lane; r < G::NR; r += 32) {
    const int gr = G::rid()[r];
    if (acc[3 * r]) atomicAdd(&p.counts[gr], acc[3 * r]);
    if (p.digests) {
      if (acc[3 * r + 1]) atomicAdd(&p.digests[2 * gr], acc[3 * r + 1]);
      if (acc[3 * r + 2]) atomicAdd(&p.digests[2 * gr + 1], acc[3 * r + 2]);
    }
  }
}

template <class G> DEV void rx_ctx_init(const RxParams &p, Ctx<G::K> &c, RxOut *o, u64 *acc, unsigned char *lb) {
  c.lane = rx_lane();
  c.o = o;
  c.walk = false;
  c.dense = p.dense != nullptr;
  c.fast = p.dense == nullptr && p.digests == nullptr && p.match_total == nullptr;
  c.acc = acc;
  c.wb = G::LIT ? lb : nullptr;
  c.ob = G::LIT ? reinterpret_cast<u32 *>(lb + 1024 * G::K) : nullptr;
  if (c.lane == 0) {
    o->acc = acc;
    o->dense = p.dense;
    o->pitch = p.pitch;
    o->gofs = p.gofs;
    o->sign = 1ull;
    o->want_digest = p.digests != nullptr;
    o->want_dense = p.dense != nullptr;
    o->rid = G::rid();
    o->status = p.status;
    o->mlist = p.matches;
    o->mcap = p.match_cap;
    o->mtotal = p.match_total;
    o->fold = nullptr;
  }
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
// tracked by an mbarrier (transaction bytes).
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

// ---------------------------------------------------------------------------
// cluster masks (bit ci = the group's factor cluster ci; G::cmask(ci) = its
// members).  The body runs exactly the clusters of its `run` mask.
// ---------------------------------------------------------------------------
template <class G> DEV u32 rx_all_clusters() { return G::NC >= 32 ? RX_FULL : ((1u << G::NC) - 1u); }
// clusters with a member in `members` (lane ci looks at cluster ci)
template <class G> DEV u32 rx_clusters_of(u32 members, u32 lane) {
  const bool hit = (int)lane < G::NC && (G::cmask((int)lane) & members) != 0u;
  return __ballot_sync(RX_FULL, hit);
}
// clusters holding a non-zero state word
template <class G> DEV u32 rx_pend_clusters(const u32 *st, u32 lane) {
  u32 pc = 0u;
  for (int s = (int)lane; s < G::NS; s += 32)
    if (st[s] != 0u) pc |= 1u << G::sci(s);
  return __reduce_or_sync(RX_FULL, pc);
}
// clusters to run in a window: a prefilter hit of a member (rmask), or --
// mode A only (not in bmc) -- carried state or no factor at all
template <class G> DEV u32 rx_run_clusters(u32 rmask, u32 bmc, u32 pendc, u32 lane) {
  const int ci = (int)lane;
  bool r = false;
  if (ci < G::NC) {
    const u32 bit = 1u << ci;
    r = (G::cmask(ci) & rmask) != 0u || (!(bmc & bit) && (((G::CALWAYS | pendc) & bit) != 0u));
  }
  return __ballot_sync(RX_FULL, r);
}

// rx_match_batch: a stream none of whose 1 KiB prefilter blocks holds a
// factor of this group (and the group has no member without a factor) has
// no match of the group and needs no state: skip it before any setup (most
// (group, packet) pairs)
// The stream is then run as an empty one (every warp of the CTA still makes
// the same runner calls: the cluster lockstep's barriers stay matched), or --
// when no warp of the CTA has work for this stream slot -- not at all.
template <class G> DEV bool rx_batch_skip(const RxParams &p, RxParams *wp) {
  if (p.len <= 0) return true;
  if (!p.pf_on || G::ALWAYS != 0u) return false;
  const u32 lane = threadIdx.x & 31u;
  const u32 *gb = p.pf_gbits + (i64)G::GID * p.pf_ntiles;
  const i64 b0 = p.pf_shift >> 10, b1 = (p.pf_shift + p.len - 1) >> 10;
  bool hit = false;
  for (i64 b = b0 + lane; b <= b1; b += 32) hit = hit || ((gb[b >> 5] >> (b & 31)) & 1u);
  if (!__any_sync(RX_FULL, hit)) {
    if (lane == 0) wp->len = wp->avail_hi = wp->valid_hi = 0;
    __syncwarp();
    return true;
  }
  return false;
}

// ---------------------------------------------------------------------------
// Dense pass 1 (no prefilter: RX_F_NO_PREFILTER or no factor at all): every
// window of the segment runs the group's whole program, gated only by the
// zero-block guards inside it (Sec. 6).  All warps of the CTA run this group
// in lockstep (one barrier per window) so that the SM fetches each line of
// the group's straight-line program once for all of them.
// ---------------------------------------------------------------------------
template <class G>
DEV void rx_run_segment_dense(const RxParams &p, int seg, RxOut *o, u64 *acc, u32 *sst, unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, o, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + G::NSMAX;
  for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
  __syncwarp();
  const RxRange ir = rx_interior(p);
  if (w_begin < w_end) rx_fetch<K>(p, ir, c.lane, xr, w_begin * Bw - Lw);
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
      G::body(c, pl, st, nst, rx_all_clusters<G>());
      u32 *t = st;
      st = nst;
      nst = t;
      __syncwarp();
    }
    __syncthreads();
  }
  if (!live) return;
  if (NS > 0 && p.seg_state) {
    u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) dst[s] = st[s];
    if (p.st_out && w_end == nwin)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
  }
  rx_flush<G>(p, c);
}

// ---------------------------------------------------------------------------
// Mode choice.  A cluster whose members all have output
// factors may run output-gated: only in windows whose frame holds one of its
// output factors, with its incoming state reconstructed on demand.  It pays
// when the input holds the output factors much more rarely than the first
// factors -- the prefilter counted both (blocks with a hit per member), so
// every warp of every kernel of this call makes the same choice.  Returns the
// mode-B clusters (bit ci).
// ---------------------------------------------------------------------------
template <class G> DEV u32 rx_mode_b(const RxParams &p, u32 lane) {
  if (!p.modeb || !p.pf_on || !p.pf_cnt || G::CBCAP == 0u) return 0u;
  const u32 *cnt = p.pf_cnt + (u64)G::GID * 64;
  const u64 nblk = (u64)p.pf_ntiles * 32;
  const bool mine = lane < (u32)G::NR;
  const u64 f = mine ? (((G::ALWAYS >> lane) & 1u) ? nblk : (u64)cnt[2 * lane]) : 0ull;
  const u64 o = mine ? (u64)cnt[2 * lane + 1] : 0ull;
  u32 bmc = 0u;
  for (int ci = 0; ci < G::NC; ++ci) {
    if (!((G::CBCAP >> ci) & 1u)) continue;
    const u32 cm = G::cmask(ci);
    const bool in = (cm >> lane) & 1u;
    u64 F = in ? f : 0ull, O = in ? o : 0ull;
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
      F += __shfl_xor_sync(RX_FULL, F, s);
      O += __shfl_xor_sync(RX_FULL, O, s);
    }
    if (6 * O + 16 < F) bmc |= 1u << ci;
  }
  return bmc;
}
// members of the clusters in `cl`
template <class G> DEV u32 rx_members_of(u32 cl, u32 lane) {
  const u32 m = ((int)lane < G::NC && ((cl >> lane) & 1u)) ? G::cmask((int)lane) : 0u;
  return __reduce_or_sync(RX_FULL, m);
}

// state words of the clusters in `cl` equal in a and b?
template <class G> DEV bool rx_state_eq_cl(const u32 *a, const u32 *b, u32 cl, u32 lane) {
  bool e = true;
  for (int s = (int)lane; s < G::NS; s += 32)
    if ((cl >> G::sci(s)) & 1u) e = e && (a[s] == b[s]);
  return __all_sync(RX_FULL, e);
}

// Mode-B walk-back: the exact incoming state of window w for the clusters in
// `stale` (cluster mask).  The group body is monotone in its incoming state
// (state streams only meet AND / OR / Advance / add-with-carry into a class),
// so running windows [w-d, w) from the zero state and from the top state
// (every carry set, every forwarded word all-ones) brackets the true state;
// once both runs agree, that is the true state.  d doubles until they agree
// or the walk reaches the stream start (state zero).  Runs are state-only
// (c.walk: no output) and execute only the stale clusters.
//
// The walk-back has its own window context and planes: they are handed to
// the out-of-line body by reference, and sharing the runner's would force
// the runner's copies into local memory for the whole segment loop.
template <class G>
__device__ __noinline__ void rx_walk_back(const RxParams &p, const RxRange &ir, const Ctx<G::K> cin, i64 w, u32 stale,
                                          u32 *st, u32 *wb, i64 len_words) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS, M = G::NSMAX;
  u32 *s0 = wb, *n0 = wb + M, *s1 = wb + 2 * M, *n1 = wb + 3 * M;
  Ctx<K> c = cin;
  u32 pl[8][K];
  u32 xr[K][8];
  c.walk = true;
  int rounds = 0;
  for (i64 d = 1;; d *= 2) {
    i64 v0 = w - d;
    const bool start = v0 <= 0;
    if (start) v0 = 0;
    for (int s = (int)c.lane; s < NS; s += 32) {
      s0[s] = 0u;
      s1[s] = (!start && ((stale >> G::sci(s)) & 1u)) ? G::top(s) : 0u;
    }
    __syncwarp();
    for (i64 v = v0; v < w; ++v) {
      const i64 fword = v * Bw - Lw;
      c.cw = (u32)((len_words - v * Bw) < Bw ? (len_words - v * Bw) : Bw);
      c.word0 = fword;
      rx_fetch<K>(p, ir, c.lane, xr, fword);
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      rx_commit_mask(p, ir, c, Lw, fword);
      rx_state_zero(n0, NS, c.lane);
      G::body(c, pl, s0, n0, stale);
      u32 *t = s0;
      s0 = n0;
      n0 = t;
      if (!start) {
        rx_state_zero(n1, NS, c.lane);
        G::body(c, pl, s1, n1, stale);
        t = s1;
        s1 = n1;
        n1 = t;
      }
      __syncwarp();
    }
    ++rounds;
    if (start || rx_state_eq_cl<G>(s0, s1, stale, c.lane)) break;
  }
  for (int s = (int)c.lane; s < NS; s += 32)
    if ((stale >> G::sci(s)) & 1u) st[s] = s0[s];
  __syncwarp();
  if (p.stats && c.lane == 0) {
    atomicAdd(&p.stats[4], 1ull);
    atomicAdd(&p.stats[5], (u64)rounds);
  }
}

// ---------------------------------------------------------------------------
// Sparse pass 1 with the prefilter (the default).  Per window the frame's
// prefilter blocks give the members whose first factor (fm) / output factor
// (om) occurs there.  Mode-A clusters run where their first factor occurs or
// state flows in; mode-B clusters run only where their output factor occurs,
// after rx_walk_back if their state is not known exactly.  Windows where
// nothing runs are skipped without loading a byte; the bytes of the window
// expected next are already in flight into a per-warp shared buffer by a TMA
// bulk copy while the body runs (a wrong guess costs a synchronous load).
// ---------------------------------------------------------------------------
#define RX_PF_BLK 1024
#define RX_PF_TILE 32768

DEV i64 rx_floor_div(i64 a, i64 b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }

template <class G>
DEV void rx_run_segment_pf(const RxParams &p, int seg, RxOut *o, u64 *acc, u32 *sst, unsigned char *tbuf, u64 *bar,
                           unsigned char *lb) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS, M = G::NSMAX;
  constexpr u32 WB = 1024u * K;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 w_begin = (i64)seg * p.sw;
  const bool live = w_begin < nwin || seg == 0;
  const i64 w_end = !live ? w_begin : (w_begin + p.sw < nwin ? w_begin + p.sw : nwin);
  Ctx<K> c;
  rx_ctx_init<G>(p, c, o, acc, lb);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *st = sst, *nst = sst + M, *wbs = sst + 2 * M;
  const u32 bmc = rx_mode_b<G>(p, c.lane);      // mode-B clusters
  const u32 bm = rx_members_of<G>(bmc, c.lane);  // ... and their members
  const u32 always_a = G::ALWAYS & ~bm;
  for (int s = (int)c.lane; s < NS; s += 32) st[s] = (seg == 0 && p.st_in) ? p.st_in[G::SBASE + s] : 0u;
  if (c.lane == 0) rx_mbar_init(bar, 1);
  __syncwarp();
  const RxRange ir = rx_interior(p);
  const u32 *gb = p.pf_gbits + (i64)G::GID * p.pf_ntiles;
  const u32 *mmf = p.pf_mmask + (i64)G::GID * 32 * p.pf_ntiles;
  const u32 *mmo = p.pf_omask ? p.pf_omask + (i64)G::GID * 32 * p.pf_ntiles : nullptr;
  auto frame_blocks = [&](i64 w, i64 &b0, i64 &b1) {
    i64 flo = (w * Bw - Lw) * 32, fhi = flo + 1024 * K;
    if (flo < p.avail_lo) flo = p.avail_lo;
    if (fhi > p.avail_hi) fhi = p.avail_hi;
    if (fhi <= flo) fhi = flo + 1;
    b0 = (flo - p.avail_lo + p.pf_shift) >> 10;
    b1 = (fhi - 1 - p.avail_lo + p.pf_shift) >> 10;
  };
  i64 bmax = 0;
  if (w_begin < w_end) {
    i64 t0;
    frame_blocks(w_end - 1, t0, bmax);
  }
  // a mode-A cluster carries state into the next window
  auto pending_a = [&](const u32 *a) -> bool {
    if (NS == 0) return false;
    return (rx_pend_clusters<G>(a, c.lane) & ~bmc) != 0u;
  };
  // first window >= w in which something must run: a block of its frame
  // holds a first factor of a mode-A member or an output factor of a mode-B
  // member (w_end if none).  Scans 32 blocks per step, one per lane: groups
  // whose mode-B members have frequent first factors have a block bit almost
  // everywhere but need to run rarely.
  auto next_hit = [&](i64 w) -> i64 {
    if (w >= w_end) return w_end;
    if (always_a != 0u) return w;
    i64 b0, b1;
    frame_blocks(w, b0, b1);
    for (i64 c0 = b0 & ~(i64)31; c0 <= bmax; c0 += 32) {
      const u32 word = gb[c0 >> 5];
      const i64 b = c0 + c.lane;
      bool need = false;
      if (((word >> c.lane) & 1u) && b >= b0 && b <= bmax)
        need = ((mmf[b] & ~bm) | (bm ? (mmo[b] & bm) : 0u)) != 0u;
      const u32 bal = __ballot_sync(RX_FULL, need);
      if (!bal) continue;
      const i64 bb = c0 + (__ffs(bal) - 1);
      if (bb <= b1) return w;
      const i64 pos = p.avail_lo + bb * RX_PF_BLK - p.pf_shift;
      const i64 wn = rx_floor_div(rx_floor_div(pos, 32) + Lw - 32 * K, Bw) + 1;
      const i64 r = wn > w + 1 ? wn : w + 1;
      return r < w_end ? r : w_end;
    }
    return w_end;
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
  u32 exact = 0u;  // mode-B clusters whose state in st[] is exact at window w
  i64 w = pending_a(st) ? w_begin : next_hit(w_begin);
  if (w < w_end) stage(w);
  // Cluster lockstep (p.lockstep): the CTA's
  // warps (one group, 16 segments) take one window each per round and then
  // walk the union of their cluster masks in ascending order with one CTA
  // barrier per cluster, so the warps that run a cluster run it together and
  // the SM fetches its straight-line code once for all of them (the
  // instruction-fetch stall, no_instructions, was the top stall of the
  // free-running form: profiles/r2_ncu_*).  Windows with nothing to run are
  // skipped between rounds without a barrier.
  u32 *const rx_cta_u = rx_cta_union();
  const bool lock = p.lockstep != 0;
  int par = 0;
  if (lock) {
    if (threadIdx.x == 0) rx_cta_u[0] = rx_cta_u[1] = 0u;
    __syncthreads();
  }
  for (;;) {
    // the next window with something to run (w_end: none left)
    u32 run = 0u, pendc = 0u;
    bool pend_in = false;
    while (w < w_end) {
      pendc = NS > 0 ? rx_pend_clusters<G>(st, c.lane) : 0u;
      pend_in = (pendc & ~bmc) != 0u;
      if (p.stats && c.lane == 0) atomicAdd(&p.stats[3], 1ull);
      i64 b0, b1;
      frame_blocks(w, b0, b1);
      u32 fmine = 0u, omine = 0u;
      for (i64 b = b0 + c.lane; b <= b1; b += 32)
        if ((gb[b >> 5] >> (b & 31)) & 1u) {
          fmine |= mmf[b];
          if (mmo) omine |= mmo[b];
        }
      const u32 fm = __reduce_or_sync(RX_FULL, fmine), om = __reduce_or_sync(RX_FULL, omine);
      const u32 rmask = (fm & ~bm) | (om & bm);
      if (rmask == 0u && !pend_in && always_a == 0u) {
        exact = 0u;
        w = next_hit(w + 1);
        continue;
      }
      // the clusters to run (never empty here: a hit, carried state or a
      // member without a factor each select a cluster)
      run = rx_run_clusters<G>(rmask, bmc, pendc, c.lane);
      if (p.stats && c.lane == 0) {
        atomicAdd(&p.stats[0], 1ull);
        atomicAdd(&p.stats[2], (u64)__popc(rmask));
        atomicAdd(&p.stats[6], (u64)__popc(run));
        u64 *gs = p.stats + 8 + 4 * G::GID;  // per group: active windows, member hits, mode-B clusters, cluster runs
        atomicAdd(&gs[0], 1ull);
        atomicAdd(&gs[1], (u64)__popc(rmask));
        gs[2] = (u64)__popc(bmc);
        atomicAdd(&gs[3], (u64)__popc(run));
      }
      break;
    }
    const bool have = w < w_end;
    const u32 runb = run & bmc;
    if (have) {
      // mode-B clusters to run whose state is stale first reconstruct it
      const u32 stale = runb & ~exact;
      if (stale) rx_walk_back<G>(p, ir, c, w, stale, st, wbs, len_words);
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
        if (staged >= 0) retire();  // a stale guess: drain it
        rx_fetch<K>(p, ir, c.lane, xr, fword);
      }
      // guess the next window and start its copy before the body runs
      if (staged < 0) stage(pend_in ? w + 1 : next_hit(w + 1));
      c.cw = (u32)((len_words - w * Bw) < Bw ? (len_words - w * Bw) : Bw);
      c.word0 = fword;
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      rx_commit_mask(p, ir, c, Lw, fword);
      if (NS > 0) rx_state_zero(nst, NS, c.lane);
    }
    // the clusters this round walks: the CTA's union (lockstep) or this
    // warp's own mask; one call site of the inlined body either way
    u32 U = run;
    if (lock) {
      if (have && c.lane == 0) atomicOr(&rx_cta_u[par], run);
      const int more = __syncthreads_or(have);
      U = rx_cta_u[par];
      // every warp read the other word before this round's barrier
      if (threadIdx.x == 0) rx_cta_u[par ^ 1] = 0u;
      par ^= 1;
      if (!more) break;
    } else if (!have) {
      break;
    }
    while (U) {
      u32 m = run;
      if (lock) {
        const u32 bit = U & (0u - U);
        U &= U - 1u;
        m = run & bit;
      } else {
        U = 0u;
      }
      if (m) G::body_i(c, pl, st, nst, m);
      if (lock && p.lockstep == 1) __syncthreads();  // 2: one barrier per round only
    }
    if (!have) continue;
    u32 *t = st;
    st = nst;
    nst = t;
    __syncwarp();
    exact = runb;  // the mode-B clusters that ran now hold their exact end state
    const i64 nw = pending_a(st) ? w + 1 : next_hit(w + 1);
    if (nw != w + 1) exact = 0u;
    w = nw;
  }
  if (staged >= 0) retire();
  if (!live) return;
  if (NS > 0 && p.seg_state) {
    // mode-B slots are not carried across segments (the next segment walks
    // back for itself): the fix-up sees zero for them on both sides
    u32 *dst = p.seg_state + ((i64)seg * G::NG + G::GID) * G::NSMAX;
    for (int s = (int)c.lane; s < NS; s += 32) dst[s] = ((bmc >> G::sci(s)) & 1u) ? 0u : st[s];
    if (p.st_out && w_end == nwin)
      for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = st[s];
  }
  rx_flush<G>(p, c);
}

// Fix-up / rematch (one warp per group): walk the windows in order carrying
// the true state; wherever it differs from the state pass 1 used, re-run the
// window with both states and apply (new - old) until they agree.  Mode-B
// clusters (exact in pass 1 already) do not run here.
template <class G>
DEV void rx_fixup_group(const RxParams &p, RxOut *o, u64 *acc, u32 *sst, unsigned char *lb, int fseg) {
  constexpr int K = G::K, Lw = G::Lw, Bw = G::Bw, NS = G::NS, M = G::NSMAX;
  if (NS == 0) return;
  const i64 len_words = rx_div_up(p.len, 32);
  const i64 nwin = rx_div_up(len_words, Bw);
  const i64 nseg = rx_div_up(nwin, p.sw);
  if (p.fix_phase == 1 && (fseg <= 0 || fseg >= nseg)) return;
  auto sstate = [&](const u32 *base, i64 seg) { return base + (seg * G::NG + G::GID) * G::NSMAX; };
  if (p.mode == 1 && p.fix_phase == 1) {
    // most segments start from a zero state: nothing to fix, leave before
    // any setup (phase 1 has a warp for every (group, segment))
    const u32 *src = sstate(p.seg_state, fseg - 1);
    bool nz = false;
    for (int s = (int)(threadIdx.x & 31u); s < NS; s += 32) nz = nz || src[s] != 0u;
    if (!__any_sync(RX_FULL, nz)) return;
  }
  Ctx<K> c;
  rx_ctx_init<G>(p, c, o, acc, lb);
  c.fast = false;  // the fix-up subtracts (sign -1) and folds match lists: rx_emit only
  // mode-B clusters were exact in pass 1 already: only the others re-run
  const u32 runa = rx_all_clusters<G>() & ~(p.mode == 1 ? rx_mode_b<G>(p, c.lane) : 0u);
  u32 pl[8][K];
  u32 xr[K][8];
  u32 *tru = sst, *old = sst + M, *t1 = sst + 2 * M, *t2 = sst + 3 * M;
  u32 fold[G::NR * K];
  if (c.lane == 0) o->fold = p.match_total ? fold : nullptr;
  __syncwarp();
  // re-run windows [w0, w1) with both states (old: the state the applied
  // results assumed, subtracted; tru: the true state, added) until the two
  // runs' states agree; returns whether they did.  part: run only the
  // clusters whose state differs between the two runs (clusters are
  // independent, so an equal state gives equal results: no difference to
  // apply); their slots then hold 0 in both runs, and `diff` ends as the
  // clusters that still differ (phase 1 takes the others' end state from
  // pass 1, which they then follow exactly)
  u32 diff = runa;
  auto walk = [&](i64 w0, i64 w1, bool part) -> bool {
    bool conv = rx_state_eq(tru, old, NS, c.lane);
    for (i64 w = w0; w < w1 && !conv; ++w) {
      if (part) {
        u32 dm = 0u;
        for (int s = (int)c.lane; s < NS; s += 32)
          if (tru[s] != old[s]) dm |= 1u << G::sci(s);
        diff = __reduce_or_sync(RX_FULL, dm) & runa;
      }
      const i64 cstart = w * Bw;
      const i64 fword = cstart - Lw;
      c.cw = (u32)((len_words - cstart) < Bw ? (len_words - cstart) : Bw);
      c.word0 = fword;
      const RxRange ir = rx_interior(p);
      rx_fetch<K>(p, ir, c.lane, xr, fword);
      rx_unpack<K>(p, ir, c, xr, pl, fword);
      rx_commit_mask(p, ir, c, Lw, fword);
      // old run: subtract
      if (c.lane == 0) {
        o->sign = ~0ull;
        o->want_dense = 0;
      }
      c.dense = false;
      if (p.match_total)  // each lane's own copy (local memory)
        for (int j = 0; j < G::NR * K; ++j) fold[j] = 0u;
      __syncwarp();
      rx_state_zero(t1, NS, c.lane);
      G::body(c, pl, old, t1, part ? diff : runa);
      // new run: add, rewrite dense words
      if (c.lane == 0) {
        o->sign = 1ull;
        o->want_dense = p.dense != nullptr;
      }
      c.dense = p.dense != nullptr;
      __syncwarp();
      rx_state_zero(t2, NS, c.lane);
      G::body(c, pl, tru, t2, part ? diff : runa);
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
    if (!walk(w_begin, w_end, true)) {
      // the segment's true end state: the walked state of the clusters that
      // still differ, pass 1's end state for the others
      const u32 *pe = sstate(p.seg_state, fseg);
      u32 *dst = p.seg_fix + (fseg * G::NG + G::GID) * G::NSMAX;
      for (int s = (int)c.lane; s < NS; s += 32) dst[s] = ((diff >> G::sci(s)) & 1u) ? tru[s] : pe[s];
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
      if (walk(w_begin, w_end, false)) {
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
  // serial form (rematch, mode 2): one warp walks the chunk carrying the true
  // state from the caller's assumed one until they agree
  for (int s = (int)c.lane; s < NS; s += 32) {
    tru[s] = p.st_in ? p.st_in[G::SBASE + s] : 0u;
    old[s] = p.st_assumed ? p.st_assumed[G::SBASE + s] : 0u;
  }
  __syncwarp();
  const bool conv = walk(0, nwin, false);
  if (p.st_out && !conv)
    for (int s = (int)c.lane; s < NS; s += 32) p.st_out[G::SBASE + s] = tru[s];
  rx_flush<G>(p, c);
}

// ---------------------------------------------------------------------------
// Cross-regex prefilter.
// One streaming pass over the input.  For every position q, x = the 4 bytes
// ending at q (little-endian, byte q on top) is tested against the anchor
// filters held in shared memory (a Bloom filter over the 4-gram anchors and,
// if the program has any, one over the 3-gram anchors and a bitmap over the
// 2-gram anchors).  Filter hits are compacted per warp and verified one per
// lane: the anchor's hash chain, then each factor's 16-byte extension window
// around q.  A tile of 32 blocks of 1 KiB is owned by one CTA, which ORs the
// member masks of the factors found into shared per-(group, block) masks
// (first / output factors apart), then writes per group one word of block
// bits, the masks of the blocks hit, and per-member block counts.
// ---------------------------------------------------------------------------
DEV u32 rx_load_u32_slow(const RxParams &p, i64 pos) {
  u32 v = 0u;
  for (int j = 0; j < 4; ++j) {
    const i64 ps = pos + j;
    if (ps >= p.avail_lo && ps < p.avail_hi) v |= (u32)p.in[ps] << (8 * j);
  }
  return v;
}

// 4 bytes ending at position base + r (0 <= r < 16) from the words w0 (bytes
// base-4..base-1) .. w4 (base+12..base+15)
DEV u32 rx_pf_x(u32 w0, u32 w1, u32 w2, u32 w3, u32 w4, int r) {
  const int m = r >> 2, s = r & 3;
  const u32 lo = m == 0 ? w0 : (m == 1 ? w1 : (m == 2 ? w2 : w3));
  const u32 hi = m == 0 ? w1 : (m == 1 ? w2 : (m == 2 ? w3 : w4));
  return s == 3 ? hi : __funnelshift_r(lo, hi, 8 * (s + 1));
}

// the 16-byte extension window of factor entry E ({ae, v[4], m[4], ...})
// for an anchor ending at q
DEV bool rx_pf_ext_ok(const RxParams &p, const u32 *E, i64 q) {
  const i64 s = q - (i64)E[0];
  u32 w[4];
  if (s - 3 >= p.avail_lo && s + 20 <= p.avail_hi) {
    const unsigned long long ad = (unsigned long long)(p.in + s);
    const u32 *al = reinterpret_cast<const u32 *>(ad & ~3ull);
    const u32 sh = (u32)(ad & 3ull) * 8u;
    const u32 x0 = __ldg(al), x1 = __ldg(al + 1), x2 = __ldg(al + 2), x3 = __ldg(al + 3), x4 = __ldg(al + 4);
    w[0] = __funnelshift_r(x0, x1, sh);
    w[1] = __funnelshift_r(x1, x2, sh);
    w[2] = __funnelshift_r(x2, x3, sh);
    w[3] = __funnelshift_r(x3, x4, sh);
  } else {
    // near the readable range's ends: a byte outside it never matches a
    // compared (masked) position
    for (int j = 0; j < 4; ++j) {
      u32 v = 0u, out = 0u;
      for (int b = 0; b < 4; ++b) {
        const i64 ps = s + 4 * j + b;
        if (ps >= p.avail_lo && ps < p.avail_hi) v |= (u32)p.in[ps] << (8 * b);
        else out |= 0xffu << (8 * b);
      }
      if (out & E[5 + j]) return false;
      w[j] = v;
    }
  }
  return ((w[0] & E[5]) == E[1]) && ((w[1] & E[6]) == E[2]) && ((w[2] & E[7]) == E[3]) && ((w[3] & E[8]) == E[4]);
}

DEV u32 rx_pf_ht_hash(u32 gram, u32 k) { return (gram ^ (k * 0x27D4EB2Fu)) * 0x9E3779B1u; }

// verify one filter hit: x = the 4 bytes ending at q, kbits: bit k-2 set if
// the k-gram filter fired.  tags: the tile's per-block direct-mapped record
// of factor entries already applied to block b (an entry seen again in the
// same block -- a common factor such as an HTTP header name -- skips its
// member-mask loop; a tag collision only costs a redundant, idempotent OR)
#define RX_PF_TAGS 64
DEV void rx_pf_verify(const RxParams &p, u32 *sm, u32 *tags, int NG, u32 x, u32 kbits, i64 q, int b) {
  const u32 *T = p.pf_tab;
  const u32 hmask = (1u << p.pf_hbits) - 1u;
  for (u32 k = 4; k >= 2; --k) {
    if (!((kbits >> (k - 2)) & 1u)) continue;
    const u32 gmask = k == 4 ? 0xffffffffu : (0xffffffffu << (8u * (4u - k)));
    const u32 gram = x & gmask;
    if (q - (i64)k + 1 < p.avail_lo) continue;
    u32 h = rx_pf_ht_hash(gram, k) >> (32u - p.pf_hbits);
    for (;;) {
      const uint4 e = __ldg(reinterpret_cast<const uint4 *>(T + p.pf_o_ht) + h);
      if (e.y == 0u) break;
      if (e.x == gram && e.y == ((k << 1) | 1u)) {
        for (u32 j = 0; j < e.w; ++j) {
          const u32 ei = e.z + j;
          u32 *tg = &tags[b * RX_PF_TAGS + (ei & (RX_PF_TAGS - 1))];
          if (*(volatile u32 *)tg == ei + 1u) continue;  // applied to this block already
          const u32 *E = T + p.pf_o_ext + 12u * ei;
          if (!rx_pf_ext_ok(p, E, q)) continue;
          const u32 t0 = __ldg(&E[9]), tn = __ldg(&E[10]);
          for (u32 t = t0; t < t0 + tn; ++t) {
            const u32 g = __ldg(&T[p.pf_o_fgent + 3 * t]), m = __ldg(&T[p.pf_o_fgent + 3 * t + 1]),
                      kind = __ldg(&T[p.pf_o_fgent + 3 * t + 2]);
            u32 *a = &sm[(kind * (u32)NG + g) * 32u + (u32)b];
            if ((*(volatile u32 *)a & m) != m) atomicOr(a, m);
          }
          *(volatile u32 *)tg = ei + 1u;
        }
      }
      h = (h + 1u) & hmask;
    }
  }
}

// smem: [filters (pf_smem_words) | member masks 2 x NG x 32 | per-warp hit
// queues 32 x 3 | factor tags 32 blocks x RX_PF_TAGS]
DEV void rx_prefilter_run(const RxParams &p, int NG) {
  extern __shared__ __align__(16) u32 pf_smem[];
  const int tid = threadIdx.x, nt = blockDim.x;
  const u32 tw = (p.pf_smem_words + 3u) & ~3u;
  u32 *tab = pf_smem;
  for (u32 i = tid; i < p.pf_smem_words; i += nt) tab[i] = __ldg(&p.pf_tab[i]);
  u32 *sm = pf_smem + tw;                      // [2][NG][32 blocks] member masks
  u32 *wq = sm + 64 * NG + 96 * (tid >> 5);   // per-warp hit queue: 32 x {offset, x, kbits}
  u32 *tags = sm + 64 * NG + 96 * (nt >> 5);   // [32 blocks][RX_PF_TAGS]
  const u32 *bl4 = tab, *bl3 = tab + p.pf_o_b3, *bg2 = tab + p.pf_o_b2;
  const bool has3 = p.pf_o_b3 != 0u, has2 = p.pf_o_b2 != 0u;
  const u32 s4 = 32u - p.pf_b4bits, s3 = 32u - p.pf_b3bits;
  const u32 lane = rx_lane();
  const i64 span = p.avail_hi - p.avail_lo;
  const i64 ntiles = (span + RX_PF_TILE - 1) / RX_PF_TILE;
  const i64 nblk = 32 * p.pf_ntiles;
  for (i64 t = blockIdx.x; t < ntiles; t += gridDim.x) {
    for (int i = tid; i < 64 * NG; i += nt) sm[i] = 0u;
    for (int i = tid; i < 32 * RX_PF_TAGS; i += nt) tags[i] = 0u;
    __syncthreads();
    const i64 tile_lo = p.avail_lo + t * RX_PF_TILE;
    // the warp's filter hits are compacted into a queue of 32 that persists
    // across the tile's chunks and is verified one hit per lane when full
    // (and once at the tile's end): full-warp verification
    u32 qn = 0;
    auto flush = [&]() {
      __syncwarp();
      if (lane < qn) {
        const u32 off = wq[3 * lane];
        rx_pf_verify(p, sm, tags, NG, wq[3 * lane + 1], wq[3 * lane + 2], tile_lo + off, (int)(off >> 10));
      }
      __syncwarp();
      qn = 0;
    };
    for (int j = 0; j < RX_PF_TILE / 16; j += nt) {
      const i64 base = tile_lo + (i64)(j + tid) * 16;
      u32 w1, w2, w3, w4;
      if (p.aligned && ((p.avail_lo & 15) == 0) && base + 16 <= p.avail_hi) {
        const uint4 v = __ldg(reinterpret_cast<const uint4 *>(p.in + base));
        w1 = v.x; w2 = v.y; w3 = v.z; w4 = v.w;
      } else {
        w1 = rx_load_u32_slow(p, base);
        w2 = rx_load_u32_slow(p, base + 4);
        w3 = rx_load_u32_slow(p, base + 8);
        w4 = rx_load_u32_slow(p, base + 12);
      }
      u32 w0 = __shfl_up_sync(RX_FULL, w4, 1);
      if (lane == 0)
        w0 = (p.aligned && ((p.avail_lo & 15) == 0) && base - 4 >= p.avail_lo && base <= p.avail_hi)
                 ? __ldg(reinterpret_cast<const u32 *>(p.in + base - 4))
                 : rx_load_u32_slow(p, base - 4);
      // filter pass over the 16 positions -> hit masks per anchor length
      // (measured: gating the Bloom tests behind a trailing-bigram bitmap
      // made the kernel slower -- most text positions pass the gate and the
      // gated loop runs divergent, profiles/r2_ncu_r2k*)
      u32 h4 = 0u, h3 = 0u, h2 = 0u;
#pragma unroll
      for (int r = 0; r < 16; ++r) {
        const u32 x = rx_pf_x(w0, w1, w2, w3, w4, r);
        const u32 a = (x * 0x9E3779B1u) >> s4;
        h4 |= ((bl4[a >> 5] >> (a & 31u)) & 1u) << r;
        if (has3) {
          const u32 b = ((x >> 8) * 0x85EBCA77u) >> s3;
          h3 |= ((bl3[b >> 5] >> (b & 31u)) & 1u) << r;
        }
        if (has2) {
          const u32 g = x >> 16;
          h2 |= ((bg2[g >> 5] >> (g & 31u)) & 1u) << r;
        }
      }
      u32 hm = h4 | h3 | h2;
      const i64 rem = p.avail_hi - base;
      if (rem < 16) hm &= rem <= 0 ? 0u : ((1u << rem) - 1u);
      for (;;) {
        const u32 bal = __ballot_sync(RX_FULL, hm != 0u);
        if (!bal) break;
        const u32 rk = __popc(bal & ((1u << lane) - 1u));
        if (hm != 0u && qn + rk < 32u) {
          const int r = __ffs(hm) - 1;
          hm &= hm - 1u;
          u32 *e = wq + 3 * (qn + rk);
          e[0] = (u32)(base + r - tile_lo);
          e[1] = rx_pf_x(w0, w1, w2, w3, w4, r);
          e[2] = ((h4 >> r) & 1u) << 2 | ((h3 >> r) & 1u) << 1 | ((h2 >> r) & 1u);
        }
        qn = qn + __popc(bal) < 32u ? qn + __popc(bal) : 32u;
        if (qn == 32u) flush();
      }
    }
    if (qn) flush();
    __syncthreads();
    // one warp per group: lane b holds block b's member masks; the group's
    // tile word of block bits is their ballot; lane m counts member m's blocks
    for (int g = tid >> 5; g < NG; g += nt >> 5) {
      const u32 f = sm[32 * g + lane], o = sm[32 * (NG + g) + lane];
      const u32 bal = __ballot_sync(RX_FULL, (f | o) != 0u);
      if (lane == 0) p.pf_gbits[(i64)g * p.pf_ntiles + t] = bal;
      if (f | o) {
        p.pf_mmask[(i64)g * nblk + t * 32 + lane] = f;
        if (p.pf_omask) p.pf_omask[(i64)g * nblk + t * 32 + lane] = o;
      }
      if (bal && p.pf_cnt) {
        u32 cf = 0u, co = 0u;
        for (int b = 0; b < 32; ++b) {
          cf += (__shfl_sync(RX_FULL, f, b) >> lane) & 1u;
          co += (__shfl_sync(RX_FULL, o, b) >> lane) & 1u;
        }
        if (cf) atomicAdd(&p.pf_cnt[(g * 32 + lane) * 2], cf);
        if (co) atomicAdd(&p.pf_cnt[(g * 32 + lane) * 2 + 1], co);
      }
    }
    __syncthreads();
  }
}
