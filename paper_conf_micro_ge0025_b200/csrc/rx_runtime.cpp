// rx_runtime.cpp -- the C ABI (include/rx.h): compile (parse -> IR -> groups
// -> CUDA C -> NVRTC sm_100a cubin, "compiled at runtime
// using NVRTC"), lazy module load, and the launches of the fused kernel.
//
// There is no CPU execution path: rx_match / rx_match_chunk / rx_rematch_chunk
// launch the generated sm_100a kernels or fail with RX_ECUDA.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvrtc.h>
#include <zlib.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <map>
#include <mutex>
#include <sstream>
#include <string>
#include <sys/stat.h>
#include <thread>
#include <unistd.h>
#include <vector>

#include "../../include/rx.h"
#include "rx_internal.h"

namespace {

thread_local std::string g_last_error;

rx_status fail(rx_status s, const std::string &m) {
  g_last_error = m;
  return s;
}

// ---------------------------------------------------------------------------
// driver entry points (no link-time libcuda dependency: the .so loads on a
// GPU-less host; module load happens at the first match)
// ---------------------------------------------------------------------------
struct Drv {
  CUresult (*ModuleLoadData)(CUmodule *, const void *) = nullptr;
  CUresult (*ModuleGetFunction)(CUfunction *, CUmodule, const char *) = nullptr;
  CUresult (*LaunchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                           CUstream, void **, void **) = nullptr;
  CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
  CUresult (*ModuleUnload)(CUmodule) = nullptr;
  CUresult (*LinkCreate)(unsigned, CUjit_option *, void **, CUlinkState *) = nullptr;
  CUresult (*LinkAddData)(CUlinkState, CUjitInputType, void *, size_t, const char *, unsigned, CUjit_option *,
                          void **) = nullptr;
  CUresult (*LinkComplete)(CUlinkState, void **, size_t *) = nullptr;
  CUresult (*LinkDestroy)(CUlinkState) = nullptr;
  bool ok = false;
  std::string why;
};

Drv &drv() {
  static Drv d;
  static std::once_flag once;
  std::call_once(once, [] {
    auto get = [](const char *name, void **fn) -> bool {
      cudaDriverEntryPointQueryResult q;
      cudaError_t e = cudaGetDriverEntryPointByVersion(name, fn, 12000, cudaEnableDefault, &q);
      return e == cudaSuccess && q == cudaDriverEntryPointSuccess && *fn;
    };
    bool ok = get("cuModuleLoadData", (void **)&d.ModuleLoadData) &&
              get("cuModuleGetFunction", (void **)&d.ModuleGetFunction) &&
              get("cuLaunchKernel", (void **)&d.LaunchKernel) &&
              get("cuFuncSetAttribute", (void **)&d.FuncSetAttribute) &&
              get("cuModuleUnload", (void **)&d.ModuleUnload) && get("cuLinkCreate", (void **)&d.LinkCreate) &&
              get("cuLinkAddData", (void **)&d.LinkAddData) && get("cuLinkComplete", (void **)&d.LinkComplete) &&
              get("cuLinkDestroy", (void **)&d.LinkDestroy);
    d.ok = ok;
    if (!ok) d.why = "CUDA driver entry points unavailable (no GPU / driver?)";
  });
  return d;
}

// ---------------------------------------------------------------------------
// cubin cache
// ---------------------------------------------------------------------------
uint64_t fnv1a(const std::string &s, uint64_t h = 1469598103934665603ull) {
  for (unsigned char c : s) {
    h ^= c;
    h *= 1099511628211ull;
  }
  return h;
}

std::string cache_dir() {
  const char *e = getenv("RX_CACHE_DIR");
  std::string d;
  if (e && *e) d = e;
  else {
    const char *h = getenv("HOME");
    d = std::string(h ? h : "/tmp") + "/.cache/bitrx";
  }
  return d;
}

void mkdirs(const std::string &d) {
  std::string cur;
  for (size_t i = 0; i < d.size(); ++i) {
    cur += d[i];
    if (d[i] == '/' && i > 0) mkdir(cur.c_str(), 0755);
  }
  mkdir(d.c_str(), 0755);
}

bool read_file(const std::string &path, std::string &out) {
  std::ifstream f(path, std::ios::binary);
  if (!f) return false;
  std::ostringstream ss;
  ss << f.rdbuf();
  out = ss.str();
  return !out.empty();
}

// gzip-compressed cache entries (cubins compress ~5x; the in-tree cache
// travels to the GPU box with the repo snapshot)
bool read_gz(const std::string &path, std::string &out) {
  gzFile f = gzopen(path.c_str(), "rb");
  if (!f) return false;
  out.clear();
  char buf[1 << 16];
  int n;
  while ((n = gzread(f, buf, sizeof buf)) > 0) out.append(buf, (size_t)n);
  const bool ok = n == 0;
  gzclose(f);
  return ok && !out.empty();
}

void write_gz_atomic(const std::string &path, const std::string &data) {
  std::string tmp = path + ".tmp" + std::to_string(getpid()) + "_" +
                    std::to_string((unsigned long long)std::hash<std::thread::id>{}(std::this_thread::get_id()));
  gzFile f = gzopen(tmp.c_str(), "wb6");
  if (!f) return;
  const bool ok = gzwrite(f, data.data(), (unsigned)data.size()) == (int)data.size();
  gzclose(f);
  if (ok) rename(tmp.c_str(), path.c_str());
  else unlink(tmp.c_str());
}

void write_file_atomic(const std::string &path, const std::string &data) {
  std::string tmp = path + ".tmp" + std::to_string(getpid()) + "_" +
                    std::to_string(std::hash<std::thread::id>()(std::this_thread::get_id()));
  {
    std::ofstream f(tmp, std::ios::binary);
    if (!f) return;
    f.write(data.data(), (std::streamsize)data.size());
  }
  rename(tmp.c_str(), path.c_str());
}

bool nvrtc_compile(const std::string &src, int max_regs, bool use_cache, std::string &cubin, std::string &log) {
  int maj = 0, mnr = 0;
  nvrtcVersion(&maj, &mnr);
  // -lineinfo only on request (RX_LINEINFO=1, for ncu source pages): in -rdc
  // mode it embeds the PTX text and makes each group unit ~4x larger
  std::vector<std::string> opts = {"--gpu-architecture=sm_100a", "-std=c++17", "-default-device", "-rdc=true",
                                   "--maxrregcount=" + std::to_string(max_regs), "-DNDEBUG"};
  const char *li = getenv("RX_LINEINFO");
  if (li && *li == '1') opts.push_back("-lineinfo");
  std::string key_src = src;
  for (auto &o : opts) key_src += "\n//" + o;
  key_src += "\n//nvrtc " + std::to_string(maj) + "." + std::to_string(mnr);
  char hex[32];
  snprintf(hex, sizeof hex, "%016llx", (unsigned long long)fnv1a(key_src));
  std::string dir = cache_dir();
  std::string path = dir + "/" + hex + ".cubin";
  if (use_cache && (read_gz(path + ".gz", cubin) || read_file(path, cubin))) return true;
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, src.c_str(), "rx_program.cu", 0, nullptr, nullptr) != NVRTC_SUCCESS) {
    log = "nvrtcCreateProgram failed";
    return false;
  }
  std::vector<const char *> ov;
  for (auto &o : opts) ov.push_back(o.c_str());
  nvrtcResult r = nvrtcCompileProgram(prog, (int)ov.size(), ov.data());
  size_t ls = 0;
  nvrtcGetProgramLogSize(prog, &ls);
  if (ls > 1) {
    log.resize(ls);
    nvrtcGetProgramLog(prog, &log[0]);
  }
  if (r != NVRTC_SUCCESS) {
    nvrtcDestroyProgram(&prog);
    return false;
  }
  size_t cs = 0;
  nvrtcGetCUBINSize(prog, &cs);
  cubin.resize(cs);
  nvrtcGetCUBIN(prog, &cubin[0]);
  nvrtcDestroyProgram(&prog);
  if (use_cache) {
    mkdirs(dir);
    write_gz_atomic(path + ".gz", cubin);
  }
  return true;
}

}  // namespace

// ---------------------------------------------------------------------------
// program
// ---------------------------------------------------------------------------
constexpr int kFixupWarps = 4;
constexpr size_t kPfTagBytes = 4 * 32 * 64;  // prefilter factor tags (RX_PF_TAGS, rx_device.cuh)
constexpr size_t kCtaHdr = 512;  // CTA header of pass 1 / fix-up shared memory (RX_CTA_HDR, rx_device.cuh)
constexpr int kPrefilterWarps = 8;
constexpr size_t kMaxSmem = 232448;  // opt-in dynamic shared memory per block (227 KB)
constexpr size_t kModuleBytes = 128u << 20;  // code per linked module (see rx_compile)
struct RxModule {
  int g_begin = 0, g_end = 0;  // group range
  int ns_max = 1, nr_max = 1;
  size_t warp_smem = 0;  // per-warp shared bytes of pass 1 / fix-up (rx_codegen.cpp warp_smem_bytes)
  bool any_state = false;
  std::string source;
  std::vector<std::string> units;  // relocatable sm_100a cubins (groups + kernels)
  // loaded (device-specific)
  int device = -1;
  CUmodule mod = nullptr;
  CUfunction pass1 = nullptr, fixup = nullptr, prefilter = nullptr;
  // prefilter tables on the device (uploaded at load)
  void *pf_mem = nullptr;
};

struct rx_program {
  rx::CompiledSet cs;
  uint32_t flags = 0;  // rx_options.flags
  int pass1_warps = 16;  // pass-1 CTA: one SM's register file at max_regs, one group (lockstep)
  std::vector<RxModule> mods;
  uint32_t n_regex = 0;
  uint32_t state_words = 0;
  uint32_t lookback = 0, lookahead = 0;
  std::string all_source;
  std::string info;
  std::mutex mu;
  // per-kernel timing (rx_set_profiling): CUDA events recorded on the launch
  // stream around every launch; kinds 0 = prefilter, 1 = pass 1, 2 = fix-up
  bool prof = false;
  struct Ev {
    int kind;
    cudaEvent_t a, b;
  };
  std::vector<Ev> prof_ev;
  double prof_ms[3] = {0, 0, 0};
  uint64_t prof_n[3] = {0, 0, 0};
  // device scratch per stream (grow-only, reused call after call): a
  // cudaMallocAsync/cudaFreeAsync pair per buffer per call left the GPU idle
  // between steps (7.5 ms per Snort-like step, 55 ms per Dotstar-like step)
  std::map<std::pair<void *, int>, std::pair<void *, size_t>> scratch;
  // rx_match_host: copy stream, staging ring and its events (lazily created)
  cudaStream_t copy_stream = nullptr;
  static constexpr int kRing = 3;
  void *ring[kRing] = {nullptr, nullptr, nullptr};
  size_t ring_bytes = 0;
  cudaEvent_t copied[kRing] = {nullptr, nullptr, nullptr}, consumed[kRing] = {nullptr, nullptr, nullptr};
  void *states[2] = {nullptr, nullptr};
  // rx_match_batch: pinned staging of the stream offsets, and the event that
  // marks the end of its last copy
  void *batch_host = nullptr;
  size_t batch_host_bytes = 0;
  cudaEvent_t batch_copied = nullptr;
};

namespace {
// scratch slots of one rx_match call
enum { SC_STATUS = 0, SC_SEGSTATE = 1, SC_PF = 2, SC_FIX = 3, SC_BATCH = 4 };
void *scratch_get(rx_program *p, cudaStream_t s, int slot, size_t bytes) {
  std::lock_guard<std::mutex> lk(p->mu);
  auto &e = p->scratch[{(void *)s, slot}];
  if (e.second < bytes) {
    if (e.first) cudaFree(e.first);  // synchronising; growth only
    e.first = nullptr;
    e.second = 0;
    if (cudaMalloc(&e.first, bytes) != cudaSuccess) return nullptr;
    e.second = bytes;
  }
  return e.first;
}
}  // namespace

extern "C" {

const char *rx_last_error(void) { return g_last_error.c_str(); }

uint32_t rx_num_regex(const rx_program *p) { return p ? p->n_regex : 0; }
uint32_t rx_num_groups(const rx_program *p) { return p ? (uint32_t)p->cs.groups.size() : 0; }
uint32_t rx_max_lookback(const rx_program *p) { return p ? p->lookback : 0; }
uint32_t rx_max_lookahead(const rx_program *p) { return p ? p->lookahead : 0; }
size_t rx_boundary_bytes(const rx_program *p) { return p ? 4 * (size_t)std::max<uint32_t>(p->state_words, 1) : 0; }
const char *rx_program_source(const rx_program *p) { return p ? p->all_source.c_str() : ""; }
uint32_t rx_kernels_per_match(const rx_program *p) {
  uint32_t n = 0;
  if (p)
    for (auto &m : p->mods) n += 1 + (m.any_state ? 2 : 0);
  if (p && p->cs.use_pf && !p->mods.empty()) n += 1;  // one prefilter pass for all modules
  return n;
}
const char *rx_program_info(const rx_program *p) { return p ? p->info.c_str() : ""; }

size_t rx_prefilter_table(const rx_program *p, const uint32_t **blob, uint32_t *hdr) {
  if (!p || !p->cs.use_pf) return 0;
  const rx::Prefilter &pf = p->cs.pf;
  if (blob) *blob = pf.blob.data();
  if (hdr) {
    const uint32_t h[12] = {pf.smem_words, pf.b4bits, pf.hbits >> 8, pf.hbits & 255u, pf.o_b3, pf.o_b2,
                            pf.o_ht,       pf.o_ext,  pf.o_fgoff,   pf.o_fgent,       (uint32_t)pf.nfactor, 0u};
    memcpy(hdr, h, sizeof h);
  }
  return pf.blob.size();
}

rx_status rx_set_profiling(rx_program *p, int on) {
  if (!p) return fail(RX_EINVAL, "null program");
  std::lock_guard<std::mutex> lk(p->mu);
  p->prof = on != 0;
  return RX_OK;
}

rx_status rx_kernel_times(rx_program *p, double *ms, uint64_t *launches, int reset) {
  if (!p) return fail(RX_EINVAL, "null program");
  std::lock_guard<std::mutex> lk(p->mu);
  for (auto &e : p->prof_ev) {
    float t = 0.f;
    if (cudaEventSynchronize(e.b) != cudaSuccess || cudaEventElapsedTime(&t, e.a, e.b) != cudaSuccess)
      return fail(RX_ECUDA, "event timing failed");
    p->prof_ms[e.kind] += t;
    p->prof_n[e.kind] += 1;
    cudaEventDestroy(e.a);
    cudaEventDestroy(e.b);
  }
  p->prof_ev.clear();
  for (int k = 0; k < 3; ++k) {
    if (ms) ms[k] = p->prof_ms[k];
    if (launches) launches[k] = p->prof_n[k];
    if (reset) {
      p->prof_ms[k] = 0;
      p->prof_n[k] = 0;
    }
  }
  return RX_OK;
}

void rx_free(rx_program *p) {
  if (!p) return;
  Drv &d = drv();
  for (auto &m : p->mods)
    if (m.mod && d.ok) {
      int cur = -1;
      cudaGetDevice(&cur);
      if (cur != m.device) cudaSetDevice(m.device);
      d.ModuleUnload(m.mod);
      if (m.pf_mem) cudaFree(m.pf_mem);
      if (cur != m.device && cur >= 0) cudaSetDevice(cur);
    }
  for (auto &kv : p->scratch)
    if (kv.second.first) cudaFree(kv.second.first);
  for (int i = 0; i < rx_program::kRing; ++i) {
    if (p->ring[i]) cudaFree(p->ring[i]);
    if (p->copied[i]) cudaEventDestroy(p->copied[i]);
    if (p->consumed[i]) cudaEventDestroy(p->consumed[i]);
  }
  for (int i = 0; i < 2; ++i)
    if (p->states[i]) cudaFree(p->states[i]);
  if (p->copy_stream) cudaStreamDestroy(p->copy_stream);
  if (p->batch_host) cudaFreeHost(p->batch_host);
  if (p->batch_copied) cudaEventDestroy(p->batch_copied);
  delete p;
}

rx_status rx_compile(const char *const *patterns, const size_t *pattern_lens, uint32_t n_patterns,
                     const rx_options *opt, rx_program **out, rx_error *err) {
  if (!out || (n_patterns && (!patterns || !pattern_lens))) return fail(RX_EINVAL, "null argument");
  *out = nullptr;
  rx_options o;
  memset(&o, 0, sizeof o);
  if (opt) o = *opt;
  rx::LowerOptions lo;
  // default 4 (the paper fixes 8; 1-4 measured ~11% faster than 8 on the Snort-like set,
  // profiles/r2_ablation_snort.md)
  lo.interval = o.interval == 0 ? 4 : (o.interval == UINT32_MAX ? 0 : (int)o.interval);
  if (o.flags & RX_F_NO_GUARDS) lo.interval = 0;
  lo.rebalance = (o.flags & RX_F_REBALANCE) && !(o.flags & RX_F_NO_REBALANCE);
  int max_regs = o.max_regs ? (int)o.max_regs : 128;

  if (o.words_per_lane != 0 && o.words_per_lane != 1 && o.words_per_lane != 2 && o.words_per_lane != 4 &&
      o.words_per_lane != 8) {
    if (err) {
      err->pattern_index = 0;
      err->byte_offset = 0;
      snprintf(err->msg, sizeof err->msg, "words_per_lane must be 0, 1, 2, 4 or 8");
    }
    return fail(RX_EINVAL, "words_per_lane must be 0, 1, 2, 4 or 8");
  }

  auto *p = new rx_program();
  p->n_regex = n_patterns;
  p->flags = o.flags;
  // pass-1 CTA size: one SM's register file (64 K registers) at max_regs
  // (rx_options.max_regs)
  max_regs = std::max(32, std::min(255, max_regs));
  // warps are allocated to the SM's four schedulers in groups of four, so a
  // CTA of 11 warps is budgeted like 12: ptxas caps an entry of 352 threads
  // at 168 registers, and a group unit compiled for 184 then fails to link
  // (measured).  Hence 16 warps up to 128 registers, 12 up to 168, else 8.
  p->pass1_warps = max_regs <= 128 ? 16 : (max_regs <= 168 ? 12 : 8);
  p->cs.pass1_warps = p->pass1_warps;
  p->cs.irs.resize(n_patterns);
  p->cs.factor_of.assign(n_patterns, -1);
  p->cs.rf.assign(n_patterns, rx::RegexFactors());
  std::vector<rx::AstP> asts(n_patterns);
  const bool use_pf = !(o.flags & RX_F_NO_PREFILTER);
  std::map<std::vector<int>, int> first_key;  // first-factor set -> clustering key
  for (uint32_t i = 0; i < n_patterns; ++i) {
    std::string pat(patterns[i], pattern_lens[i]);
    rx::ParseError pe;
    rx::AstP ast = rx::parse_regex(pat, pe);
    if (!ast || pe.code) {
      if (err) {
        err->pattern_index = i;
        err->byte_offset = (uint32_t)pe.at;
        snprintf(err->msg, sizeof err->msg, "%s", pe.msg.c_str());
      }
      delete p;
      return fail((rx_status)pe.code, "pattern " + std::to_string(i) + ": " + pe.msg);
    }
    if (rx::ast_expanded_size(*ast) > 20000) {
      if (err) {
        err->pattern_index = i;
        err->byte_offset = 0;
        snprintf(err->msg, sizeof err->msg, "expansion too large");
      }
      delete p;
      return fail(RX_ETOOBIG, "pattern " + std::to_string(i) + ": expansion too large");
    }
    if (use_pf) {
      rx::regex_factors(*ast, p->cs, p->cs.rf[i]);
      if (!(o.flags & RX_F_MODEB) || (o.flags & RX_F_NO_MODEB)) p->cs.rf[i].out.clear();
      const auto &fs = p->cs.rf[i].first;
      if (!fs.empty()) {
        auto it = first_key.find(fs);
        const int key = it == first_key.end() ? (int)first_key.size() : it->second;
        if (it == first_key.end()) first_key[fs] = key;
        p->cs.factor_of[i] = key;
      }
    }
    {
      rx::LowerOptions ro = lo;
      ro.lead_noguard = use_pf && p->cs.factor_of[i] >= 0;
      rx::lower_regex(*ast, ro, p->cs.irs[i]);
    }
    if (lo.rebalance) rx::rebalance_regex(p->cs.irs[i]);
    std::string why;
    if (!rx::analyze_regex(p->cs.irs[i], why)) {
      delete p;
      return fail(RX_EUNSUPPORTED, why);
    }
    asts[i] = std::move(ast);
  }
  std::string why;
  if (!rx::plan_groups(p->cs, (int)o.group_size, (int)o.words_per_lane, why)) {
    if (err) {
      err->pattern_index = 0;
      err->byte_offset = 0;
      snprintf(err->msg, sizeof err->msg, "%s", why.c_str());
    }
    delete p;
    return fail(RX_ETOOBIG, why);
  }
  p->cs.use_pf = use_pf && !p->cs.factors.empty();
  if (!p->cs.use_pf)  // no factor at all: every group runs dense, nothing is output-gated
    for (auto &rf : p->cs.rf) rf = rx::RegexFactors();
  {
    std::vector<const rx::Ast *> ap;
    for (auto &a : asts) ap.push_back(a.get());
    rx::LowerOptions co = lo;
    co.lead_noguard = p->cs.use_pf;
    if (!rx::build_clusters(p->cs, ap, co, why)) {
      delete p;
      return fail(RX_EUNSUPPORTED, why);
    }
  }
  if (p->cs.use_pf) rx::build_prefilter(p->cs);
  // one relocatable NVRTC unit per group + the kernel unit, compiled in
  // parallel and linked into one module by nvJitLink
  int G = (int)p->cs.groups.size();
  unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  std::ostringstream info;
  uint32_t sbase = 0;
  RxModule mm;
  mm.g_begin = 0;
  mm.g_end = G;
  for (int gi = 0; gi < G; ++gi) {
    auto &g = p->cs.groups[gi];
    info << "group " << gi << ": regexes=" << g.regexes.size() << " K=" << g.K << " Lw=" << g.Lw << " Rw=" << g.Rw
         << " Bw=" << g.Bw << " slots=" << g.nslots << " clusters=" << g.clusters.size() << " members=";
    for (size_t m = 0; m < g.regexes.size(); ++m) info << (m ? "," : "") << g.regexes[m];
    info << "\n";
    p->lookback = std::max<uint32_t>(p->lookback, 32u * (uint32_t)g.Lw);
    p->lookahead = std::max<uint32_t>(p->lookahead, 32u * (uint32_t)g.Rw);
    mm.ns_max = std::max(mm.ns_max, g.nslots);
    mm.nr_max = std::max<int>(mm.nr_max, (int)g.regexes.size());
    if (g.nslots > 0) mm.any_state = true;
    sbase += (uint32_t)g.nslots;
  }
  p->state_words = sbase;
  info << "prefilter: " << (p->cs.use_pf ? "on" : "off") << ", factors=" << p->cs.factors.size() << "\n";
  for (uint32_t i = 0; i < n_patterns; ++i) {
    info << "regex " << i << ": factor ";
    if (p->cs.use_pf) info << rx::factor_info(p->cs, (int)i);
    else info << "none (always runs)";
    info << "\n" << rx::dump_ir(p->cs.irs[i]);
  }
  // shared memory: pass 1 / fix-up per warp, prefilter per CTA (ADVICE r1:
  // a program whose layout exceeds the opt-in limit must fail here, not at
  // every launch)
  mm.warp_smem = rx::warp_smem_bytes(p->cs);
  if (mm.warp_smem * p->pass1_warps + kCtaHdr > kMaxSmem) {
    const size_t need = mm.warp_smem * p->pass1_warps + kCtaHdr;
    delete p;
    return fail(RX_ETOOBIG, "pass-1 shared memory " + std::to_string(need) + " B exceeds the 227 KB per-block limit (fewer state slots / regexes per group, or "
                                "smaller words_per_lane)");
  }
  if (p->cs.use_pf) {
    const size_t pfb =
        4 * (((size_t)p->cs.pf.smem_words + 3) & ~(size_t)3) + 4 * 64 * (size_t)G + 4 * 96 * kPrefilterWarps +
        kPfTagBytes;
    if (pfb > kMaxSmem) {
      delete p;
      return fail(RX_ETOOBIG, "prefilter shared memory " + std::to_string(pfb) + " B exceeds the 227 KB limit");
    }
  }
  p->info = info.str();
  // one relocatable NVRTC unit per group, compiled in parallel; then the
  // groups are split into modules of at most kModuleBytes of code (the
  // driver's linker crashed in cuLinkComplete on one image of all 545 group
  // units of the 10k-regex set), each with its own kernel unit
  bool use_cache = !(o.flags & RX_F_NO_CACHE);
  auto compile_all = [&](std::vector<std::string> &srcs, std::vector<std::string> &cubins,
                         std::vector<std::string> &logs) -> bool {
    cubins.assign(srcs.size(), std::string());
    logs.assign(srcs.size(), std::string());
    std::vector<int> okv(srcs.size(), 0);
    std::vector<std::thread> th;
    std::atomic<size_t> next{0};
    size_t nthreads = std::min<size_t>(srcs.size(), hw);
    for (size_t t = 0; t < nthreads; ++t)
      th.emplace_back([&] {
        for (;;) {
          size_t m = next++;
          if (m >= srcs.size()) break;
          okv[m] = nvrtc_compile(srcs[m], max_regs, use_cache, cubins[m], logs[m]) ? 1 : 0;
        }
      });
    for (auto &t : th) t.join();
    for (size_t m = 0; m < srcs.size(); ++m) {
      if (!okv[m]) {
        std::string head = logs[m].substr(0, 240);
        if (err) {
          err->pattern_index = 0;
          err->byte_offset = 0;
          snprintf(err->msg, sizeof err->msg, "%s", head.c_str());
        }
        fail(RX_EJIT, "NVRTC: " + logs[m].substr(0, 4000));
        return false;
      }
    }
    return true;
  };
  std::vector<std::string> gsrc(G), gcub, glog;
  for (int gi = 0; gi < G; ++gi) gsrc[gi] = rx::emit_group_unit(p->cs, gi);
  if (!compile_all(gsrc, gcub, glog)) {
    delete p;
    return RX_EJIT;
  }
  std::vector<std::pair<int, int>> ranges;
  {
    size_t acc = 0;
    int b = 0;
    for (int gi = 0; gi < G; ++gi) {
      if (gi > b && acc + gcub[gi].size() > kModuleBytes) {
        ranges.push_back({b, gi});
        b = gi;
        acc = 0;
      }
      acc += gcub[gi].size();
    }
    if (G > 0 || ranges.empty()) ranges.push_back({b, G});
  }
  std::vector<std::string> ksrc(ranges.size()), kcub, klog;
  for (size_t m = 0; m < ranges.size(); ++m) ksrc[m] = rx::emit_kernel_unit(p->cs, ranges[m].first, ranges[m].second);
  if (!compile_all(ksrc, kcub, klog)) {
    delete p;
    return RX_EJIT;
  }
  for (int gi = 0; gi < G; ++gi) p->all_source += gsrc[gi];
  for (size_t m = 0; m < ranges.size(); ++m) {
    RxModule mod;
    mod.g_begin = ranges[m].first;
    mod.g_end = ranges[m].second;
    mod.warp_smem = mm.warp_smem;
    for (int gi = mod.g_begin; gi < mod.g_end; ++gi) {
      const auto &g = p->cs.groups[gi];
      mod.ns_max = std::max(mod.ns_max, g.nslots);
      mod.nr_max = std::max<int>(mod.nr_max, (int)g.regexes.size());
      if (g.nslots > 0) mod.any_state = true;
      mod.units.push_back(std::move(gcub[gi]));
    }
    mod.units.push_back(std::move(kcub[m]));  // relocatable; linked by the driver at module load
    p->all_source += ksrc[m];
    p->mods.push_back(std::move(mod));
  }
  p->info += "modules: " + std::to_string(ranges.size()) + " (code MB:";
  for (auto &m : p->mods) {
    size_t b = 0;
    for (auto &u : m.units) b += u.size();
    p->info += " " + std::to_string(b >> 20);
  }
  p->info += ")\n";
  *out = p;
  return RX_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------
// launch
// ---------------------------------------------------------------------------
namespace {

struct RxParamsHost {  // must mirror RxParams in rx_device.cuh (tests/test_library_cpu.py checks the fields)
  const unsigned char *in;
  long long avail_lo, avail_hi;
  long long valid_lo, valid_hi;
  long long len;
  long long gofs;
  unsigned long long *counts;
  unsigned long long *digests;
  unsigned int *dense;
  unsigned long long pitch;
  unsigned int *status;
  unsigned int *seg_state;
  const unsigned int *st_in;
  unsigned int *st_out;
  const unsigned int *st_assumed;
  int sw;
  int nseg_max;
  int aligned;
  int mode;
  int accumulate;
  int modeb;
  int lockstep;
  const unsigned int *pf_tab;
  unsigned int pf_words, pf_smem_words;
  unsigned int pf_b4bits, pf_b3bits, pf_hbits;
  unsigned int pf_o_b3, pf_o_b2, pf_o_ht, pf_o_ext, pf_o_fgoff, pf_o_fgent;
  unsigned int *pf_gbits;
  unsigned int *pf_mmask;
  unsigned int *pf_omask;
  unsigned int *pf_cnt;
  long long pf_ntiles;
  int pf_on;
  unsigned long long *stats;
  unsigned long long *matches;
  unsigned long long match_cap;
  unsigned long long *match_total;
  int fix_phase;
  unsigned int *seg_fix;
  unsigned int *seg_nc;
  const unsigned long long *batch_off;
  long long batch_n;
  long long batch_spw;
  long long pf_shift;
};

rx_status ensure_loaded(rx_program *p, int &device) {
  Drv &d = drv();
  if (cudaGetDevice(&device) != cudaSuccess) return fail(RX_ECUDA, "no CUDA device");
  if (!d.ok) return fail(RX_ECUDA, d.why);
  std::lock_guard<std::mutex> lk(p->mu);
  for (auto &m : p->mods) {
    if (m.mod && m.device == device) continue;
    if (m.mod) return fail(RX_EINVAL, "program was loaded on another device; compile one program per device");
    cudaFree(nullptr);  // make the primary context current
    // link the relocatable units (SASS already: no JIT) into one image
    char lerr[4096];
    lerr[0] = 0;
    CUjit_option lo[] = {CU_JIT_ERROR_LOG_BUFFER, CU_JIT_ERROR_LOG_BUFFER_SIZE_BYTES};
    void *lv[] = {(void *)lerr, (void *)(uintptr_t)sizeof lerr};
    CUlinkState ls;
    CUresult r = d.LinkCreate(2, lo, lv, &ls);
    if (r != CUDA_SUCCESS) return fail(RX_ECUDA, "cuLinkCreate failed: " + std::to_string((int)r));
    for (size_t u = 0; u < m.units.size() && r == CUDA_SUCCESS; ++u) {
      std::string nm = "unit" + std::to_string(u) + ".cubin";
      r = d.LinkAddData(ls, CU_JIT_INPUT_CUBIN, (void *)m.units[u].data(), m.units[u].size(), nm.c_str(), 0, nullptr,
                        nullptr);
    }
    void *img = nullptr;
    size_t img_size = 0;
    if (r == CUDA_SUCCESS) r = d.LinkComplete(ls, &img, &img_size);
    if (r == CUDA_SUCCESS) r = d.ModuleLoadData(&m.mod, img);
    d.LinkDestroy(ls);
    if (r != CUDA_SUCCESS)
      return fail(RX_ECUDA, "link/load of the program failed: " + std::to_string((int)r) + " " + lerr);
    if (d.ModuleGetFunction(&m.pass1, m.mod, "rx_pass1") != CUDA_SUCCESS ||
        d.ModuleGetFunction(&m.fixup, m.mod, "rx_fixup") != CUDA_SUCCESS)
      return fail(RX_ECUDA, "kernel symbols missing");
    if (p->cs.use_pf) {
      if (d.ModuleGetFunction(&m.prefilter, m.mod, "rx_prefilter") != CUDA_SUCCESS)
        return fail(RX_ECUDA, "rx_prefilter symbol missing");
      const rx::Prefilter &pf = p->cs.pf;
      if (cudaMalloc(&m.pf_mem, 4 * pf.blob.size() + 16) != cudaSuccess) return fail(RX_ENOMEM, "prefilter tables");
      if (cudaMemcpy(m.pf_mem, pf.blob.data(), 4 * pf.blob.size(), cudaMemcpyHostToDevice) != cudaSuccess)
        return fail(RX_ECUDA, "prefilter table upload");
    }
    m.device = device;
  }
  return RX_OK;
}

rx_status launch(rx_program *p, RxModule &m, CUfunction f, long long blocks, int warps_per_block,
                 const RxParamsHost &prm, cudaStream_t s) {
  Drv &d = drv();
  if (blocks <= 0) return RX_OK;
  if (blocks > 0x7fffffffLL) return fail(RX_EINVAL, "grid too large");
  // shared memory: pass 1 / fix-up = per-warp layout of rx_codegen.cpp
  // emit_group_unit; prefilter = [filters | 2 x NG x 32 member masks | hit queues]
  size_t bytes = kCtaHdr + (size_t)warps_per_block * m.warp_smem;
  if (f == m.prefilter)
    bytes = 4 * (((size_t)prm.pf_smem_words + 3) & ~(size_t)3) + 4 * 64 * p->cs.groups.size() +
            4 * 96 * (size_t)warps_per_block + kPfTagBytes;
  if (bytes > kMaxSmem) return fail(RX_ETOOBIG, "shared memory layout exceeds 227 KB");
  const unsigned smem = (unsigned)bytes;
  if (smem > 48 * 1024 &&
      d.FuncSetAttribute(f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)smem) != CUDA_SUCCESS)
    return fail(RX_ECUDA, "cuFuncSetAttribute(max dynamic shared memory = " + std::to_string(smem) + ") failed");
  bool prof;
  {
    std::lock_guard<std::mutex> lk(p->mu);
    prof = p->prof;
  }
  rx_program::Ev ev{f == m.prefilter ? 0 : (f == m.pass1 ? 1 : 2), nullptr, nullptr};
  if (prof) {
    cudaEventCreate(&ev.a);
    cudaEventCreate(&ev.b);
    cudaEventRecord(ev.a, s);
  }
  RxParamsHost local = prm;
  void *args[] = {&local};
  CUresult r =
      d.LaunchKernel(f, (unsigned)blocks, 1, 1, 32 * warps_per_block, 1, 1, smem, (CUstream)s, args, nullptr);
  if (prof) {
    cudaEventRecord(ev.b, s);
    std::lock_guard<std::mutex> lk(p->mu);
    p->prof_ev.push_back(ev);
  }
  if (r != CUDA_SUCCESS) return fail(RX_ECUDA, "cuLaunchKernel failed: " + std::to_string((int)r));
  return RX_OK;
}

long long div_up(long long a, long long b) { return (a + b - 1) / b; }

// batch: rx_match_batch -- d_input/len span all streams back to back, the
// per-stream outputs are laid out by stream, `batch_off` (device) holds the
// n_streams + 1 offsets; one launch sequence for all streams
struct BatchArg {
  const unsigned long long *d_off;
  long long n;
  long long max_len;  // longest stream (bytes)
};

rx_status run(rx_program *p, const uint8_t *d_input, uint64_t len, uint64_t halo_left, uint64_t halo_right,
              uint64_t gofs, const void *st_in, void *st_out, const void *st_assumed, int accumulate, int mode,
              cudaStream_t stream, const rx_output *out, const BatchArg *batch = nullptr) {
  if (!p || !out || !out->d_counts) return fail(RX_EINVAL, "null argument");
  if (len && !d_input) return fail(RX_EINVAL, "null input");
  if (!batch && out->d_bitstreams && out->pitch_words < (len + 31) / 32)
    return fail(RX_EINVAL, "pitch_words too small");
  if ((halo_left != 0 && halo_left < p->lookback) || (halo_right != 0 && halo_right < p->lookahead))
    return fail(RX_EINVAL, "halo smaller than rx_max_lookback / rx_max_lookahead");
  if (out->d_matches && !out->d_match_total) return fail(RX_EINVAL, "d_matches needs d_match_total");
  int device = -1;
  rx_status s = ensure_loaded(p, device);
  if (s != RX_OK) return s;
  const uint32_t n = p->n_regex;
  if (!accumulate && mode != 2) {
    if (n && cudaMemsetAsync(out->d_counts, 0, 8ull * n, stream) != cudaSuccess) return fail(RX_ECUDA, "memset");
    if (n && out->d_digests && cudaMemsetAsync(out->d_digests, 0, 16ull * n, stream) != cudaSuccess)
      return fail(RX_ECUDA, "memset");
    if (n && out->d_bitstreams &&
        cudaMemsetAsync(out->d_bitstreams, 0, 4ull * n * out->pitch_words, stream) != cudaSuccess)
      return fail(RX_ECUDA, "memset");
    if (out->d_status && cudaMemsetAsync(out->d_status, 0, 4, stream) != cudaSuccess) return fail(RX_ECUDA, "memset");
    if (out->d_match_total && cudaMemsetAsync(out->d_match_total, 0, 8, stream) != cudaSuccess)
      return fail(RX_ECUDA, "memset");
  }
  RxParamsHost prm;
  memset(&prm, 0, sizeof prm);
  prm.in = d_input;
  prm.avail_lo = -(long long)halo_left;
  prm.avail_hi = (long long)(len + halo_right);
  // valid stream bytes: a chunk's halo holds real bytes; the stream start
  // (no halo) has none before position 0
  prm.valid_lo = -(long long)halo_left;
  prm.valid_hi = (long long)(len + halo_right);
  prm.len = (long long)len;
  prm.gofs = (long long)gofs;
  prm.counts = (unsigned long long *)out->d_counts;
  prm.digests = (unsigned long long *)out->d_digests;
  prm.dense = out->d_bitstreams;
  prm.pitch = out->pitch_words;
  prm.status = out->d_status;
  prm.st_in = (const unsigned int *)st_in;
  prm.st_out = (unsigned int *)st_out;
  prm.st_assumed = (const unsigned int *)st_assumed;
  prm.aligned = (((uintptr_t)d_input) & 15) == 0 ? 1 : 0;
  prm.accumulate = accumulate;
  prm.matches = (unsigned long long *)out->d_matches;
  prm.match_cap = out->d_matches ? out->match_cap : 0;
  prm.match_total = (unsigned long long *)out->d_match_total;
  // mode B (output-gated clusters) only for a whole
  // stream: its walk-back may read any earlier byte and reconstructs state
  // from the stream start, so chunks (incoming / outgoing state) use mode A
  prm.modeb = (mode == 0 && !st_in && !st_out && halo_left == 0) ? 1 : 0;
  prm.lockstep = (p->flags & RX_F_NO_LOCKSTEP) ? 0 : ((p->flags & RX_F_LOCKSTEP_ROUND) ? 2 : 1);
  if (!prm.status) {
    unsigned int *status_scratch = (unsigned int *)scratch_get(p, stream, SC_STATUS, 256);
    if (!status_scratch) return fail(RX_ENOMEM, "status");
    cudaMemsetAsync(status_scratch, 0, 4, stream);
    prm.status = status_scratch;
  }
  const long long len_words = div_up((long long)len, 32);
  if (mode == 2) {
    prm.mode = 2;
    prm.sw = 1 << 30;
    prm.nseg_max = 1;
    for (auto &m : p->mods) {
      if (!m.any_state) continue;
      prm.seg_state = nullptr;
      s = launch(p, m, m.fixup, div_up(m.g_end - m.g_begin, kFixupWarps), kFixupWarps, prm, stream);
      if (s != RX_OK) return s;
    }
    return RX_OK;
  }
  // pass-1 geometry: CTAs of 16 warps, one group per CTA, 16 consecutive
  // segments; ~16 waves of 148 CTAs so that the hardware CTA scheduler
  // evens out the data-dependent work
  const int G = (int)p->cs.groups.size();
  long long max_nwin = 0;
  for (auto &g : p->cs.groups) max_nwin = std::max(max_nwin, div_up(len_words, g.Bw));
  const long long waves = 16;
  const long long target_ctas = 148LL * waves;
  const long long cpg0 = std::max<long long>(1, div_up(target_ctas, std::max(G, 1)));
  long long sw = std::max<long long>(4, div_up(max_nwin, cpg0 * p->pass1_warps));
  long long nseg_max = std::max<long long>(1, div_up(max_nwin, sw));
  if (batch) {
    // pass-1 "segment" s = streams [s*spw, (s+1)*spw), each run whole by the
    // segment's warp one after the other (no fix-up); spw sized for ~16 waves
    const long long spw = std::max<long long>(1, div_up(batch->n, cpg0 * p->pass1_warps));
    // windows of the longest stream (the dense runner's lockstep loop count)
    int min_bw = 1 << 30;
    for (auto &g : p->cs.groups) min_bw = std::min(min_bw, g.Bw);
    sw = std::max<long long>(1, div_up(div_up(batch->max_len, 32), std::max(min_bw, 1)));
    nseg_max = std::max<long long>(1, div_up(batch->n, spw));
    prm.batch_off = batch->d_off;
    prm.batch_n = batch->n;
    prm.batch_spw = spw;
    prm.modeb = 0;
  }
  const long long cpg = div_up(nseg_max, p->pass1_warps);
  prm.sw = (int)std::min<long long>(sw, 1 << 30);
  prm.nseg_max = (int)nseg_max;
  prm.mode = 0;
  const bool stats_on = (p->flags & RX_F_STATS) != 0;
  // scratch indexed by global group id (group units use G::NG, G::GID and the
  // program-wide NSMAX): sized for all groups, shared by the modules
  int ns_all = 1;
  bool any_state = false;
  for (auto &m : p->mods) {
    ns_all = std::max(ns_all, m.ns_max);
    any_state = any_state || m.any_state;
  }
  const size_t bytes = 4ull * (size_t)nseg_max * (size_t)G * (size_t)ns_all;
  unsigned int *seg_state = nullptr;
  if (batch) any_state = false;  // whole streams per warp: nothing to fix up
  if (any_state && !(seg_state = (unsigned int *)scratch_get(p, stream, SC_SEGSTATE, bytes)))
    return fail(RX_ENOMEM, "seg_state");
  prm.seg_state = seg_state;
  prm.mode = 0;
  prm.pf_on = 0;
  if (p->cs.use_pf) {
    // one prefilter pass for all groups (module 0 holds the kernel; it
    // indexes its outputs by global group id)
    const long long span = prm.avail_hi - prm.avail_lo;
    const long long ntiles = std::max<long long>(1, div_up(span, 32768));
    const size_t gb_bytes = ((size_t)4 * (size_t)ntiles * (size_t)G + 255) & ~(size_t)255;
    const size_t bl_bytes = ((size_t)4 * 32 * (size_t)ntiles * (size_t)G + 255) & ~(size_t)255;
    const size_t cnt_bytes = (size_t)4 * 64 * (size_t)G;
    // output-factor masks only if some regex has output factors (mode B)
    bool any_out = false;
    for (auto &rf : p->cs.rf) any_out = any_out || !rf.out.empty();
    const size_t ob_bytes = any_out ? bl_bytes : 0;
    char *pf_scratch = (char *)scratch_get(p, stream, SC_PF, gb_bytes + bl_bytes + ob_bytes + cnt_bytes + 256);
    if (!pf_scratch) return fail(RX_ENOMEM, "prefilter scratch");
    const rx::Prefilter &pf = p->cs.pf;
    RxModule &m0 = p->mods[0];
    prm.pf_tab = (const unsigned int *)m0.pf_mem;
    prm.pf_words = (unsigned int)pf.blob.size();
    prm.pf_smem_words = pf.smem_words;
    prm.pf_b4bits = pf.b4bits;
    prm.pf_b3bits = pf.hbits >> 8;
    prm.pf_hbits = pf.hbits & 255u;
    prm.pf_o_b3 = pf.o_b3;
    prm.pf_o_b2 = pf.o_b2;
    prm.pf_o_ht = pf.o_ht;
    prm.pf_o_ext = pf.o_ext;
    prm.pf_o_fgoff = pf.o_fgoff;
    prm.pf_o_fgent = pf.o_fgent;
    prm.pf_gbits = (unsigned int *)pf_scratch;
    prm.pf_mmask = (unsigned int *)(pf_scratch + gb_bytes);
    prm.pf_omask = any_out ? (unsigned int *)(pf_scratch + gb_bytes + bl_bytes) : nullptr;
    // per-member block counts feed only the mode-B choice
    prm.pf_cnt = any_out ? (unsigned int *)(pf_scratch + gb_bytes + bl_bytes + ob_bytes) : nullptr;
    prm.pf_ntiles = ntiles;
    prm.pf_on = 1;
    if (prm.pf_cnt && cudaMemsetAsync(prm.pf_cnt, 0, cnt_bytes, stream) != cudaSuccess)
      return fail(RX_ECUDA, "memset");
    // 8-warp CTAs, several per SM (the verification of filter hits is a
    // chain of dependent loads: more resident warps hide it)
    s = launch(p, m0, m0.prefilter, std::min<long long>(ntiles, 148LL * 8), kPrefilterWarps, prm, stream);
    if (s != RX_OK) return s;
  }
  unsigned long long *stats = nullptr;
  const size_t stats_bytes = 8 * (8 + 4 * (size_t)G);
  if (stats_on && cudaMalloc((void **)&stats, stats_bytes) == cudaSuccess) cudaMemsetAsync(stats, 0, stats_bytes, stream);
  for (auto &m : p->mods) {
    const int mg = m.g_end - m.g_begin;
    prm.mode = 0;
    prm.stats = stats;
    s = launch(p, m, m.pass1, cpg * mg, p->pass1_warps, prm, stream);
    prm.stats = nullptr;
    if (s != RX_OK) break;
  }
  if (stats) {
    std::vector<unsigned long long> h(stats_bytes / 8);
    cudaMemcpyAsync(h.data(), stats, stats_bytes, cudaMemcpyDeviceToHost, stream);
    cudaStreamSynchronize(stream);
    fprintf(stderr, "[rx stats] groups=%d window_visits=%llu active=%llu member_hits=%llu walkbacks=%llu "
            "walk_rounds=%llu cluster_runs=%llu\n", G, h[3], h[0], h[2], h[4], h[5], h[6]);
    for (int g = 0; g < G; ++g)
      fprintf(stderr, "[rx stats] group %d: active=%llu member_hits=%llu modeB_members=%llu cluster_runs=%llu\n", g,
              h[8 + 4 * g], h[9 + 4 * g], h[10 + 4 * g], h[11 + 4 * g]);
    cudaFree(stats);
  }
  if (s != RX_OK) return s;
  if (any_state) {
    // carry fix-up, phase 1: one warp per (group, segment) in parallel;
    // phase 2: one warp per group, only where a segment's carry outlived it.
    // (pf_on stays set: the fix-up recomputes the mode-B choice from the
    // prefilter's counts and leaves those clusters alone)
    prm.mode = 1;
    void *fx = nullptr;
    const size_t nc_bytes = 4ull * (size_t)nseg_max * (size_t)G;
    if (!(fx = scratch_get(p, stream, SC_FIX, bytes + nc_bytes + 256))) return fail(RX_ENOMEM, "fix-up scratch");
    prm.seg_fix = (unsigned int *)fx;
    prm.seg_nc = (unsigned int *)((char *)fx + ((bytes + 255) & ~(size_t)255));
    cudaMemsetAsync(prm.seg_nc, 0, nc_bytes, stream);
    for (int phase = 1; phase <= 2 && s == RX_OK; ++phase) {
      prm.fix_phase = phase;
      for (auto &m : p->mods) {
        if (!m.any_state) continue;
        const long long mg = m.g_end - m.g_begin;
        s = launch(p, m, m.fixup, div_up(phase == 1 ? mg * nseg_max : mg, kFixupWarps), kFixupWarps, prm, stream);
        if (s != RX_OK) break;
      }
    }
    prm.fix_phase = 0;
    if (s != RX_OK) return s;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(RX_ECUDA, cudaGetErrorString(e));
  return RX_OK;
}

}  // namespace

extern "C" {

rx_status rx_match(const rx_program *p, const uint8_t *d_input, uint64_t len, void *stream, const rx_output *out) {
  return run(const_cast<rx_program *>(p), d_input, len, 0, 0, 0, nullptr, nullptr, nullptr, 0, 0,
             (cudaStream_t)stream, out);
}

rx_status rx_match_chunk(const rx_program *p, const uint8_t *d_input, uint64_t len, uint64_t halo_left,
                         uint64_t halo_right, uint64_t global_offset, const void *d_state_in, void *d_state_out,
                         int accumulate, void *stream, const rx_output *out) {
  return run(const_cast<rx_program *>(p), d_input, len, halo_left, halo_right, global_offset, d_state_in,
             d_state_out, nullptr, accumulate, 0, (cudaStream_t)stream, out);
}

rx_status rx_rematch_chunk(const rx_program *p, const uint8_t *d_input, uint64_t len, uint64_t halo_left,
                           uint64_t halo_right, uint64_t global_offset, const void *d_state_assumed,
                           const void *d_state_true, void *d_state_out, void *stream, const rx_output *out) {
  return run(const_cast<rx_program *>(p), d_input, len, halo_left, halo_right, global_offset, d_state_true,
             d_state_out, d_state_assumed, 1, 2, (cudaStream_t)stream, out);
}


// SURVEY 8(f) N3 / P:L178 (MIMD: many independent input streams).  Stream i
// is d_input[offsets[i] .. offsets[i+1]) and is matched as a whole input of
// its own (zero state at its start, nothing readable past either end), so
// no match and no state crosses a stream boundary.  One launch sequence for
// the whole batch: one prefilter pass over the concatenation (a factor
// straddling two streams is only a false positive), then pass 1 with one
// warp per (group, stream) running the stream whole (rx_batch_view).
rx_status rx_match_batch(const rx_program *p, const uint8_t *d_input, const uint64_t *offsets, uint32_t n_streams,
                         void *stream, const rx_output *out) {
  if (!p || !out || !out->d_counts || (n_streams && !offsets)) return fail(RX_EINVAL, "null argument");
  uint64_t max_len = 0;
  for (uint32_t i = 0; i < n_streams; i++) {
    if (offsets[i + 1] < offsets[i]) return fail(RX_EINVAL, "offsets must be non-decreasing");
    max_len = std::max<uint64_t>(max_len, offsets[i + 1] - offsets[i]);
  }
  if (out->d_bitstreams && out->pitch_words < (max_len + 31) / 32) return fail(RX_EINVAL, "pitch_words too small");
  if (n_streams && offsets[n_streams] && !d_input) return fail(RX_EINVAL, "null input");
  cudaStream_t st = (cudaStream_t)stream;
  const uint64_t n = p->n_regex;
  const uint64_t ns = n_streams;
  if (n && ns && cudaMemsetAsync(out->d_counts, 0, 8ull * n * ns, st) != cudaSuccess) return fail(RX_ECUDA, "memset");
  if (n && ns && out->d_digests && cudaMemsetAsync(out->d_digests, 0, 16ull * n * ns, st) != cudaSuccess)
    return fail(RX_ECUDA, "memset");
  if (n && ns && out->d_bitstreams &&
      cudaMemsetAsync(out->d_bitstreams, 0, 4ull * n * ns * out->pitch_words, st) != cudaSuccess)
    return fail(RX_ECUDA, "memset");
  if (out->d_status && cudaMemsetAsync(out->d_status, 0, 4, st) != cudaSuccess) return fail(RX_ECUDA, "memset");
  if (out->d_match_total && cudaMemsetAsync(out->d_match_total, 0, 8, st) != cudaSuccess)
    return fail(RX_ECUDA, "memset");
  if (!ns) return RX_OK;
  const uint64_t total = offsets[ns] - offsets[0];
  // the offsets, rebased to offsets[0], on the device (stream-ordered copy
  // from a program-owned pinned staging buffer)
  rx_program *pm = const_cast<rx_program *>(p);
  const size_t obytes = 8ull * (ns + 1);
  unsigned long long *d_off = (unsigned long long *)scratch_get(pm, st, SC_BATCH, obytes);
  if (!d_off) return fail(RX_ENOMEM, "batch offsets");
  unsigned long long *h_off = nullptr;
  {
    std::lock_guard<std::mutex> lk(pm->mu);
    // the previous batch's offsets copy must have read the staging buffer
    // before it is rewritten (an event, not a stream synchronisation)
    if (pm->batch_copied) cudaEventSynchronize(pm->batch_copied);
    else if (cudaEventCreateWithFlags(&pm->batch_copied, cudaEventDisableTiming) != cudaSuccess)
      return fail(RX_ECUDA, "event");
    if (pm->batch_host_bytes < obytes) {
      if (pm->batch_host) cudaFreeHost(pm->batch_host);
      pm->batch_host = nullptr;
      pm->batch_host_bytes = 0;
      if (cudaMallocHost(&pm->batch_host, obytes) != cudaSuccess) return fail(RX_ENOMEM, "batch offsets (host)");
      pm->batch_host_bytes = obytes;
    }
    h_off = (unsigned long long *)pm->batch_host;
    for (uint64_t i = 0; i <= ns; ++i) h_off[i] = offsets[i] - offsets[0];
    if (cudaMemcpyAsync(d_off, h_off, obytes, cudaMemcpyHostToDevice, st) != cudaSuccess ||
        cudaEventRecord(pm->batch_copied, st) != cudaSuccess)
      return fail(RX_ECUDA, "offsets copy");
  }
  BatchArg b{d_off, (long long)ns, (long long)max_len};
  // the streams' match-list positions and digests are relative to d_input
  return run(pm, d_input + offsets[0], total, 0, 0, offsets[0], nullptr, nullptr, nullptr, 1, 0, st, out, &b);
}

rx_status rx_match_host(const rx_program *pc, const uint8_t *h_input, uint64_t len, uint64_t piece_bytes,
                        void *stream, const rx_output *out) {
  rx_program *p = const_cast<rx_program *>(pc);
  if (!p || !out || !out->d_counts) return fail(RX_EINVAL, "null argument");
  if (len && !h_input) return fail(RX_EINVAL, "null input");
  if (out->d_bitstreams && out->pitch_words < (len + 31) / 32) return fail(RX_EINVAL, "pitch_words too small");
  uint64_t P = piece_bytes ? piece_bytes : (64ull << 20);  // measured: 32 / 64 / 128 MiB -> 21.8 / 27.2 / 23.4 GB/s e2e
  P = (P + 1023) & ~1023ull;
  const uint64_t hl = p->lookback, hr = p->lookahead;
  const size_t need = (size_t)(P + hl + hr + 64);
  const size_t sbytes = std::max<size_t>(4, 4 * (size_t)p->state_words);
  cudaStream_t s = (cudaStream_t)stream;
  {
    std::lock_guard<std::mutex> lk(p->mu);
    if (!p->copy_stream && cudaStreamCreateWithFlags(&p->copy_stream, cudaStreamNonBlocking) != cudaSuccess)
      return fail(RX_ECUDA, "copy stream");
    if (p->ring_bytes < need) {
      cudaDeviceSynchronize();  // growth only
      for (int i = 0; i < rx_program::kRing; ++i) {
        if (p->ring[i]) cudaFree(p->ring[i]);
        p->ring[i] = nullptr;
        if (cudaMalloc(&p->ring[i], need) != cudaSuccess) return fail(RX_ENOMEM, "staging buffers");
        if (!p->copied[i] && (cudaEventCreateWithFlags(&p->copied[i], cudaEventDisableTiming) != cudaSuccess ||
                              cudaEventCreateWithFlags(&p->consumed[i], cudaEventDisableTiming) != cudaSuccess))
          return fail(RX_ECUDA, "events");
      }
      p->ring_bytes = need;
    }
    for (int i = 0; i < 2; ++i)
      if (!p->states[i] && cudaMalloc(&p->states[i], sbytes) != cudaSuccess) return fail(RX_ENOMEM, "state buffers");
  }
  if (len == 0) return rx_match(p, nullptr, 0, stream, out);
  const uint64_t npieces = (len + P - 1) / P;
  for (uint64_t i = 0; i < npieces; ++i) {
    const int b = (int)(i % rx_program::kRing);
    const uint64_t a = i * P, e = std::min(len, a + P);
    const uint64_t lo = a >= hl ? a - hl : 0, hi = std::min(len, e + hr);
    // the copy into ring slot b waits until the match that last read it is done
    if (i >= (uint64_t)rx_program::kRing && cudaStreamWaitEvent(p->copy_stream, p->consumed[b], 0) != cudaSuccess)
      return fail(RX_ECUDA, "wait");
    if (cudaMemcpyAsync(p->ring[b], h_input + lo, hi - lo, cudaMemcpyHostToDevice, p->copy_stream) != cudaSuccess)
      return fail(RX_ECUDA, "host-to-device copy");
    if (cudaEventRecord(p->copied[b], p->copy_stream) != cudaSuccess ||
        cudaStreamWaitEvent(s, p->copied[b], 0) != cudaSuccess)
      return fail(RX_ECUDA, "event");
    rx_output o = *out;
    if (out->d_bitstreams) o.d_bitstreams = out->d_bitstreams + a / 32;  // a is a multiple of 1 KiB
    const void *st_in = i == 0 ? nullptr : p->states[(i + 1) & 1];
    void *st_out = p->states[i & 1];
    rx_status r = run(p, (const uint8_t *)p->ring[b] + (a - lo), e - a, a - lo, hi - e, a, st_in, st_out, nullptr,
                      i == 0 ? 0 : 1, 0, s, &o);
    if (r != RX_OK) return r;
    if (cudaEventRecord(p->consumed[b], s) != cudaSuccess) return fail(RX_ECUDA, "event");
  }
  return RX_OK;
}

}  // extern "C"
