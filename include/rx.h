/*
 * rx.h -- C ABI of the B200-native interleaved bitstream regex engine.
 *
 * The operation (PAPER.md = /root/reference/PAPER.md; "P:Lnnn" = its line):
 *   a set of regular expressions is "evaluated concurrently over a shared
 *   input stream" (Sec. 3.1); for each regex r the result is the
 *   match-end bitstream S_r, "a 1 at position i indicates a successful match
 *   ending at that position" under all-match semantics (Sec. 2), plus
 *   per-regex match counts (the paper validates "match positions and counts",
 *   P:L401).  Precisely: S_r[i] = 1 iff some s <= i has input[s..i] in L(r)
 *   (non-empty, unanchored; DESIGN.md "Readings" c1-c17).
 *
 * How: rx_compile lowers patterns to a Parabix-style bitstream IR
 * (CC from 8 basis streams, AND/OR/NOT, Advance, MatchStar, while -- Fig. 2,
 * P:L77-116; Listing 3), groups regexes and
 * JIT-compiles one fused interleaved sm_100a kernel (Sec. 3.3)
 * with NVRTC.  rx_match launches it; no CPU fallback exists -- every
 * function that computes returns RX_ECUDA when no CUDA device is usable.
 *
 * Conventions
 *  - All pointers named d_* are DEVICE pointers (cudaMalloc / torch CUDA
 *    tensors).  The caller owns the input and every output buffer; the
 *    library owns the program and its scratch (stream-ordered).
 *  - Calls that take a stream are asynchronous: they return a launch status;
 *    device-side conditions are reported in out->d_status.
 *  - Positions are 64-bit (inputs may exceed 2^32 bytes).
 *  - Thread safety: distinct (rx_program, stream) pairs may be used
 *    concurrently from different host threads.
 */
#ifndef RX_H_
#define RX_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct rx_program rx_program; /* opaque: host IR + loaded sm_100a module */

typedef enum {
  RX_OK = 0,
  RX_EPARSE = 1,       /* pattern syntax error (err->pattern_index / byte_offset) */
  RX_EUNSUPPORTED = 2, /* anchors, backreferences, lookaround, lazy quantifiers */
  RX_ETOOBIG = 3,      /* expansion of R{n,m} or program size over the caps */
  RX_EJIT = 4,         /* NVRTC / module load failure (err->msg has the log head) */
  RX_ECUDA = 5,        /* CUDA runtime error or no usable device */
  RX_EINVAL = 6,       /* bad argument (NULL, misaligned, too small) */
  RX_ENOMEM = 7,
  RX_EOVERFLOW = 8
} rx_status;

typedef struct {
  uint32_t pattern_index; /* which pattern failed */
  uint32_t byte_offset;   /* where in it */
  char msg[256];
} rx_error;

/* Tunables.  Defaults follow the paper's fixed defaults (merge size 8,
 * interval size 8, CTA count 256, max registers 128) where they apply. */
typedef struct {
  uint32_t interval;       /* zero-block-skipping guard interval in IR instructions (Sec. 6); 0 = default 4 (the paper: 8); UINT32_MAX = no guards */
  uint32_t max_regs;       /* NVRTC --maxrregcount; 0 = default 128 */
  uint32_t group_size;     /* max regexes per group; 0 = auto */
  uint32_t words_per_lane; /* K: 32-bit words per lane per window (window = 1024*K positions): 0 (auto), 1, 2, 4
                              or 8; anything else is RX_EINVAL */
  uint32_t flags;          /* RX_F_* below */
  uint32_t reserved[3];
} rx_options;

#define RX_F_NO_REBALANCE 1u /* force Shift Rebalancing off */
#define RX_F_REBALANCE 8u    /* enable Shift Rebalancing (Sec. 5); off by default: on B200 it buys
                                ILP only (no shift barriers at warp scope) -- see DESIGN.md */
#define RX_F_NO_GUARDS 2u    /* disable Zero Block Skipping (Sec. 6) */
#define RX_F_NO_CACHE 4u     /* do not read/write the on-disk cubin cache */
#define RX_F_NO_PREFILTER 16u /* disable the cross-regex literal prefilter: every group
                                 runs every window, gated only by Zero Block Skipping (Sec. 6) */
#define RX_F_NO_MODEB 32u     /* accepted for compatibility: mode B is off unless RX_F_MODEB */
#define RX_F_MODEB 256u       /* allow output-gated clusters: a cluster whose members all have
                                 output factors may run only where one occurs, reconstructing its incoming state by a
                                 walk-back.  Off by default: measured slower on the Snort-like set (ablation ladder,
                                 profiles/r2_ablation_snort.md) */
#define RX_F_NO_LOCKSTEP 128u /* sparse pass 1 without cluster lockstep: each warp runs its own windows'
                                 clusters freely (ablation) */
#define RX_F_LOCKSTEP_ROUND 512u /* cluster lockstep with one CTA barrier per window round instead of one per
                                   cluster (experiment) */
#define RX_F_STATS 64u        /* debug: count visited / active windows and walk-backs per rx_match and print
                                 them to stderr (synchronises the stream; not for timing) */

/* Compile n patterns (byte strings, not NUL-terminated).  On error returns
 * the status and, if err != NULL, fills it.  *out owns everything. */
rx_status rx_compile(const char *const *patterns, const size_t *pattern_lens, uint32_t n_patterns,
                     const rx_options *opt /* nullable */, rx_program **out, rx_error *err /* nullable */);
void rx_free(rx_program *p);

uint32_t rx_num_regex(const rx_program *p);
uint32_t rx_num_groups(const rx_program *p);
/* Static halo in bytes a chunk needs before / after its committed range
 * (DESIGN.md "Margins"): unbounded constructs are carried in the boundary
 * state instead. */
uint32_t rx_max_lookback(const rx_program *p);
uint32_t rx_max_lookahead(const rx_program *p);
/* Bytes of boundary state (MatchStar carries, forwarded loop tails). */
size_t rx_boundary_bytes(const rx_program *p);
/* Number of this library's kernels one rx_match launches (pass 1 + fix-up). */
uint32_t rx_kernels_per_match(const rx_program *p);
/* The generated CUDA C source of the program (NUL-terminated, owned by p). */
const char *rx_program_source(const rx_program *p);
/* Human-readable IR / per-group geometry dump (owned by p). */
const char *rx_program_info(const rx_program *p);
/* The prefilter's device table (host copy, owned by p; layout documented in
 * rx_prefilter.cpp build_prefilter) and its header words hdr[12] = {smem
 * words, log2 bits of the 4-gram Bloom filter, of the 3-gram one, of the
 * anchor hash, offsets of the 3-gram filter, the 2-gram bitmap, the hash, the
 * extension entries, the factor->group ranges and triples, #factors, 0}.
 * Returns the table's size in u32 words (0: no prefilter).  For tests and
 * analysis; matching never needs it. */
size_t rx_prefilter_table(const rx_program *p, const uint32_t **blob, uint32_t *hdr /* [12], nullable */);

typedef struct {
  uint32_t regex;
  uint32_t pad;
  uint64_t pos;
} rx_match_t;

typedef struct {
  uint64_t *d_counts;     /* required: u64[n_regex], OVERWRITTEN with the match counts */
  uint64_t *d_digests;    /* nullable: u64[2*n_regex]: sum splitmix64(p), sum splitmix64(p^0x9E3779B97F4A7C15) */
  uint32_t *d_bitstreams; /* nullable: u32[n_regex * pitch_words], LSB-first (bit p of word p/32); bits >= len are 0 */
  uint64_t pitch_words;   /* >= ceil(len/32) when d_bitstreams != NULL */
  uint32_t *d_status;     /* nullable: u32 device flags, bit0 = iteration cap hit (result not exact),
                             bit2 = a fix-up run lost a match the speculative run listed (never expected:
                             match sets are monotone in the incoming state) */
  /* Compacted match list ("match positions"): one entry per set bit of
   * every S_r, {regex id, global position}, in no particular order.  Both
   * nullable; d_matches requires d_match_total.  *d_match_total receives the
   * true number of matches (zeroed unless accumulating); entries beyond
   * match_cap are dropped, so a caller seeing total > cap re-runs with a
   * larger list.  With d_match_total alone the total is counted only. */
  rx_match_t *d_matches;
  uint64_t match_cap;
  uint64_t *d_match_total;
} rx_output;

/* Match the whole input d_input[0..len).  Asynchronous on `stream`
 * (a cudaStream_t; NULL = legacy default stream). */
rx_status rx_match(const rx_program *p, const uint8_t *d_input, uint64_t len, void *stream, const rx_output *out);

/* Chunked / multi-GPU form: commit positions [0, len) of a chunk whose bytes
 * are readable at d_input[-halo_left .. len + halo_right).  Positions in the
 * match list and the digests are global_offset + i (so digests of chunks add
 * up to the whole stream's); bitstreams stay chunk-relative.
 * d_state_in: nullable device blob of rx_boundary_bytes() (NULL = the chunk
 * starts the stream: zero state); d_state_out: nullable, receives the state
 * at the chunk end.  Counts/digests are ACCUMULATED when `accumulate` != 0. */
rx_status rx_match_chunk(const rx_program *p, const uint8_t *d_input, uint64_t len, uint64_t halo_left,
                         uint64_t halo_right, uint64_t global_offset, const void *d_state_in, void *d_state_out,
                         int accumulate, void *stream, const rx_output *out);

/* Correction for a chunk that was matched assuming d_state_assumed but whose
 * true incoming state is d_state_true: re-runs windows from the chunk start
 * until the two runs' states agree, adding (new - old) to counts/digests and
 * rewriting bitstream words.  d_state_out receives the corrected end state
 * (or is left untouched when the runs converge before the end). */
rx_status rx_rematch_chunk(const rx_program *p, const uint8_t *d_input, uint64_t len, uint64_t halo_left,
                           uint64_t halo_right, uint64_t global_offset, const void *d_state_assumed,
                           const void *d_state_true, void *d_state_out, void *stream, const rx_output *out);

/* MIMD form ("a set of regular expressions ... over
 * a shared input stream", extended to many independent streams, e.g. one per
 * packet flow).  offsets: HOST u64[n_streams + 1], non-decreasing; stream i is
 * d_input[offsets[i] .. offsets[i+1]) and is matched as a complete input of
 * its own: zero state at its start, no byte of a neighbouring stream is ever
 * read, so no match crosses a stream boundary.  Outputs are per stream:
 * d_counts u64[n_streams][n_regex], d_digests u64[n_streams][n_regex][2]
 * (over positions relative to d_input, like the match list), d_bitstreams u32[n_streams][n_regex][pitch]
 * (pitch_words >= ceil(max stream length / 32); stream-relative bits); the
 * match list is shared and holds positions relative to d_input (offsets[i] + i-th byte), so the stream
 * of an entry is found by searching offsets.  All OVERWRITTEN.  Empty streams
 * are valid.  Errors: RX_EINVAL for null pointers, decreasing offsets or a
 * short pitch (nothing launched).  Asynchronous on `stream`; this first form
 * issues one launch sequence per non-empty stream. */
rx_status rx_match_batch(const rx_program *p, const uint8_t *d_input, const uint64_t *offsets, uint32_t n_streams,
                         void *stream, const rx_output *out);

/* Whole stream from HOST memory, end to end: the input is copied to the
 * device in pieces of piece_bytes (0 = 64 MiB; rounded up to a multiple of
 * 1 KiB) on an internal copy stream, and piece i is matched with
 * rx_match_chunk while piece i+1 is in flight.  Pieces are matched in order on
 * `stream`, each with rx_max_lookback bytes of the previous piece as its left
 * halo, rx_max_lookahead bytes of the next as its right halo and the previous
 * piece's end state as its exact incoming state, so the result equals
 * rx_match over the whole stream (counts, digests, match list; dense words
 * at their stream positions).  h_input should be page-locked (cudaHostAlloc /
 * cudaHostRegister) for the copies to overlap; pageable memory works but
 * serialises them.  Device staging buffers are owned by the program (reused
 * call after call).  Outputs are OVERWRITTEN.  Asynchronous on `stream`:
 * h_input must stay valid and unmodified until the stream reaches the end of
 * the call's work.  Errors as rx_match, RX_ENOMEM for the staging buffers. */
rx_status rx_match_host(const rx_program *p, const uint8_t *h_input, uint64_t len, uint64_t piece_bytes, void *stream,
                        const rx_output *out);

/* Per-kernel device timing (for roofline reporting): when on, every launch
 * of the program is bracketed by CUDA events on its stream.  rx_kernel_times
 * waits for the recorded events and writes the accumulated milliseconds and
 * launch counts of the three kernels, ms[0..2] / launches[0..2] = prefilter,
 * pass 1 (the fused interleaved kernel), fix-up; reset != 0 zeroes them. */
rx_status rx_set_profiling(rx_program *p, int on);
rx_status rx_kernel_times(rx_program *p, double *ms /* [3], nullable */, uint64_t *launches /* [3], nullable */,
                          int reset);

/* Last error message of this thread (static storage). */
const char *rx_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* RX_H_ */
