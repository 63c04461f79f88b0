// bcf_capi.cu -- the C ABI (include/bcf.h): argument checking, the pass
// driver of the pairwise mergesort, temp sizing,
// launch dispatch over the instantiated (E, u) set, the distributed-sort
// helper kernels and the optional per-kernel event profiler.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/bcf.h"
#include "bcf_kernels.cuh"
#include "bcf_launch.h"

namespace bcf {
namespace setops {
cudaError_t make_tags(uint32_t* ta, long long na, uint32_t* tb, long long nb, cudaStream_t s);
cudaError_t compact(int op, const uint32_t* M, const uint32_t* V, long long n, unsigned long long* counts,
                    unsigned long long* d_count, uint32_t* out, uint32_t* out_src, cudaStream_t s);
long long compact_blocks(long long n);
}
namespace wc {
bool generate_host(uint32_t* out, uint64_t n, int E, int u, uint64_t seed);
cudaError_t generate_device(uint32_t* out, uint64_t n, int E, int u, uint64_t seed, cudaStream_t s, bool* ok);
}

// ---------------------------------------------------------------------------
// launch table
// ---------------------------------------------------------------------------
LaunchTable& launch_table() {
  static LaunchTable* t = [] {
    auto* p = new LaunchTable();
    register_E7(*p);
    register_E8(*p);
    register_E9(*p);
    register_E10(*p);
    register_E11(*p);
    register_E12(*p);
    register_E13(*p);
    register_E14(*p);
    register_E15(*p);
    register_E16(*p);
    register_E17(*p);
    register_E31(*p);
    return p;
  }();
  return *t;
}

// Defaults for sm_100a (measured by the E/u sweep):
// E = 31 is coprime with w = 32 (rho = identity, TMA-staged tiles) and
// E + 1 = 32 makes the in-register merge one 32-wide bitonic merger; u = 128
// keeps the tile (3968 keys) and the per-thread registers within budget.
static constexpr int DEFAULT_E = 31;
static constexpr int DEFAULT_U = 128;
// Pairs carry a value and a tag per register: E = 31 spills the register
// budget; with pairs merge passes on the window kernel, (11, 256) is the
// measured best of the pairs sweep at 2^26 (profiles/r01_pairs_sweep_window_2p26.txt:
// 5.22 ms vs 5.47 at (17, 256), the previous default under the TMA kernel).
static constexpr int DEFAULT_E_PAIRS = 11;
static constexpr int DEFAULT_U_PAIRS = 256;

// ---------------------------------------------------------------------------
// errors, profiler, launch accounting
// ---------------------------------------------------------------------------
static thread_local int t_last_cuda_error = 0;
static std::atomic<long long> g_launches{0};
static std::atomic<int> g_prof_on{0};
static std::mutex g_prof_mu;

struct ProfRec {
  const char* name;
  cudaEvent_t a, b;
  uint64_t keys;
};
static std::vector<ProfRec> g_recs;
static std::vector<cudaEvent_t> g_pool;

static cudaEvent_t pool_get() {
  cudaEvent_t e = nullptr;
  if (!g_pool.empty()) {
    e = g_pool.back();
    g_pool.pop_back();
    return e;
  }
  cudaEventCreate(&e);
  return e;
}

static bcf_status cuda_fail(cudaError_t e) {
  t_last_cuda_error = (int)e;
  return BCF_ERROR_CUDA;
}

template <class F>
static cudaError_t launch(const char* name, uint64_t keys, cudaStream_t s, F&& f) {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  if (!g_prof_on.load(std::memory_order_relaxed)) return f();
  cudaEvent_t a, b;
  {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    a = pool_get();
    b = pool_get();
  }
  cudaEventRecord(a, s);
  cudaError_t e = f();
  cudaEventRecord(b, s);
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_recs.push_back({name, a, b, keys});
  return e;
}

struct Params {
  int E, U, algo;
};

static bcf_status resolve(const bcf_params* p, Params& out, bool pairs) {
  out.E = (p && p->items_per_thread) ? p->items_per_thread : (pairs ? DEFAULT_E_PAIRS : DEFAULT_E);
  out.U = (p && p->block_threads) ? p->block_threads : (pairs ? DEFAULT_U_PAIRS : DEFAULT_U);
  out.algo = p ? p->algo : BCF_ALGO_CONFLICT_FREE;
  if (out.algo != BCF_ALGO_CONFLICT_FREE && out.algo != BCF_ALGO_BASELINE) return BCF_ERROR_INVALID_VALUE;
  if (out.E < E_MIN || out.E > E_MAX || (out.E > 17 && out.E != 31) || u_index(out.U) < 0)
    return BCF_ERROR_UNSUPPORTED;
  return BCF_SUCCESS;
}

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// threads per block-sort tile (a power-of-two multiple of u; BCF_BS_SAME=1
// keeps the block sort at u, for A/B measurements)
static int bs_threads(const Params& p, bool cf, bool pairs) {
  static const bool same = [] {
    const char* v = getenv("BCF_BS_SAME");
    return v && v[0] == '1';
  }();
  static const int forced = [] {
    const char* v = getenv("BCF_BS_THREADS");
    return v ? atoi(v) : 0;
  }();
  if (forced && cf && !pairs && p.E == 31 && u_index(forced) >= 0 && forced >= p.U) return forced;
  if (cf && !pairs && p.E == 31 && p.U == 128 && !same) return 256;
  return p.U;
}

// Two-tile block sort (keys-only CF at E = 31, block tiles of 256 threads):
// runs of 2 x 7936 keys, one merge pass fewer.  Opt-in, BCF_BS2=1
// (read per call): measured slower at 2^24, the extra shared-memory level
// costs 35 us against the 30 us merge pass it saves
// (profiles/r02_ab_block_sort2_2p24.txt).
static bool bs2_enabled() {
  const char* v = getenv("BCF_BS2");
  return v && v[0] == '1';
}
static bool use_bs2(const Params& p, bool cf, bool pairs, int Ubs) {
  if (!cf || pairs || !bs2_enabled() || Ubs != 256) return false;
  const Variant& v = launch_table().v[p.E][u_index(Ubs)][0][0];
  return v.block_sort2 != nullptr;
}

// BCF_TRACE=<pass>: record a per-CTA timeline of that merge pass (debug)
static unsigned long long* g_trace = nullptr;
static const size_t TRACE_WORDS = 1 << 21;
static int trace_pass_wanted() {
  static const int want = [] {
    const char* v = getenv("BCF_TRACE");
    return v ? atoi(v) : -1;
  }();
  return want;
}
static bool trace_requested() { return trace_pass_wanted() >= 0; }
// BCF_TRACE_MULTI=1: per-CTA, per-pass timeline of the multi-pass launch
// (slots 4p: wait start, 4p+1: inputs ready, 4p+2: pass published)
static unsigned long long* trace_buffer();
static unsigned long long* multi_trace() {
  static const bool on = [] {
    const char* v = getenv("BCF_TRACE_MULTI");
    return v && v[0] == '1';
  }();
  return on ? trace_buffer() : nullptr;
}
static unsigned long long* trace_buffer() {
  if (!g_trace) {
    if (cudaMalloc(&g_trace, TRACE_WORDS * 8) != cudaSuccess) return nullptr;
    cudaMemset(g_trace, 0, TRACE_WORDS * 8);
  }
  return g_trace;
}
static unsigned long long* trace_for_pass(int pass) {
  if (pass != trace_pass_wanted()) return nullptr;
  return trace_buffer();
}

// BCF_MULTI=1: every merge pass of a sort in one persistent launch (dataflow
// between passes through per-CTA progress flags) instead of one launch per
// pass.  Off by default: measured slower at 2^24 (0.551 vs 0.517 ms per sort,
// profiles/r02_trace_multipass_2p24.txt): per-CTA pass times vary ~2.5x and
// the dependency chains accumulate that spread, while the per-pass launches
// overlap through PDL.
static bool multipass_disabled() {
  static const bool off = [] {
    const char* v = getenv("BCF_MULTI");
    return !(v && v[0] == '1');
  }();
  return off;
}
static constexpr int MAX_PROGRESS_CTAS = 2048;  // 1536 per-CTA flags + 512 per-pass counters

// BCF_ONE_CTA_PER_SM=1 (measurement mode for the unit-level bank-conflict
// counter): LSU-only kernels (block sort and the plain merge kernel, no bulk
// copies) with one CTA per SM looping over tiles.  ncu's
// l1tex__data_bank_conflicts_pipe_lsu_mem_shared also counts ~6 store
// wavefronts per CTA launched onto an SM that runs other CTAs, and port
// arbitration between STS and async copies (tools/ncu_calib_lsu.cu); this mode
// has neither, so the counter measures address conflicts alone.
static bool one_cta_per_sm() {
  static const bool on = [] {
    const char* v = getenv("BCF_ONE_CTA_PER_SM");
    return v && v[0] == '1';
  }();
  return on;
}
static long long sm_count() {
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

// BCF_NO_TMA=1 selects the non-persistent merge kernel (A/B measurements)
static bool tma_disabled() {
  static const bool off = [] {
    const char* v = getenv("BCF_NO_TMA");
    return (v && v[0] == '1') || one_cta_per_sm();
  }();
  return off;
}

// ---------------------------------------------------------------------------
// the pairwise mergesort driver
//   block sort: tiles of T = U*E -> runs of T (run r descending iff r odd, CF)
//   pass i = 1..P: runs of R = T*2^(i-1) merged pairwise; pass P writes d_out
// buffers: buf[0] = out, buf[1] = temp; the block sort writes buf[P % 2] and
// pass i writes buf[(P - i) % 2], so the last pass lands in out.
// ---------------------------------------------------------------------------
static bcf_status sort_impl(const uint32_t* in_k, uint32_t* out_k, const uint32_t* in_v, uint32_t* out_v,
                            uint64_t n, void* d_temp, size_t* temp_bytes, const bcf_params* pp,
                            cudaStream_t s, bool f32, bool pairs) {
  if (!temp_bytes) return BCF_ERROR_INVALID_VALUE;
  Params p;
  bcf_status st = resolve(pp, p, pairs);
  if (st != BCF_SUCCESS) return st;
  if (pairs && p.algo == BCF_ALGO_BASELINE) return BCF_ERROR_UNSUPPORTED;
  // two ping-pong buffers X, Y (256-B aligned, 64 words of slack for the
  // sigma-shifted descending runs); only the final pass writes d_out
  const size_t key_bytes = align_up(((size_t)n + 64) * sizeof(uint32_t), 256);
  // + per-CTA progress flags of the multi-pass merge launch
  const size_t need = 256 + key_bytes * 2 * (pairs ? 2 : 1) + MAX_PROGRESS_CTAS * sizeof(unsigned);
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return BCF_SUCCESS;
  }
  if (*temp_bytes < need) return BCF_ERROR_TEMP_TOO_SMALL;
  if (n == 0) return BCF_SUCCESS;
  if (!in_k || !out_k || (pairs && (!in_v || !out_v))) return BCF_ERROR_INVALID_VALUE;
  if (n > (1ull << 33)) return BCF_ERROR_UNSUPPORTED;

  const Variant& var = launch_table().v[p.E][u_index(p.U)][p.algo][pairs ? 1 : 0];
  if (!var.block_sort || !var.merge) return BCF_ERROR_UNSUPPORTED;
  const bool cf = p.algo == BCF_ALGO_CONFLICT_FREE;
  // Block-sort tile: keys-only CF at E = 31 sorts tiles of 2u threads (its
  // first five levels run in registers across the warp, so one more shared
  // level costs less than the merge pass it saves); merge passes keep u.
  const int Ubs = bs_threads(p, cf, pairs);
  const Variant& vbs = launch_table().v[p.E][u_index(Ubs)][p.algo][pairs ? 1 : 0];
  if (!vbs.block_sort) return BCF_ERROR_UNSUPPORTED;
  const bool one_sm = one_cta_per_sm();
  const bool bs2 = !one_sm && use_bs2(p, cf, pairs, Ubs);
  const long long T = (long long)p.U * p.E;
  const long long Tbs = (long long)Ubs * p.E * (bs2 ? 2 : 1);  // the block sort's run length
  const long long tiles = (long long)((n + T - 1) / T);
  const long long tiles_bs = (long long)((n + Tbs - 1) / Tbs);
  int lg_bs = 0;  // log2(Tbs / T)
  while ((T << lg_bs) < Tbs) ++lg_bs;
  int P = 0;
  while ((Tbs << P) < (long long)n) ++P;
#if defined(BCF_TIMING_SKIP_LEVELS) || defined(BCF_TIMING_SKIP_WARP) || defined(BCF_TIMING_BS_ONLY)
  P = 0;  // timing-only builds: the block sort alone
#endif
  const bool use_tma = cf && var.merge_tma != nullptr && !tma_disabled();

  char* tb = (char*)align_up((size_t)d_temp, 256);
  uint32_t* X = (uint32_t*)tb;
  uint32_t* Y = (uint32_t*)(tb + key_bytes);
  uint32_t* XV = pairs ? (uint32_t*)(tb + 2 * key_bytes) : nullptr;
  uint32_t* YV = pairs ? (uint32_t*)(tb + 3 * key_bytes) : nullptr;

  unsigned* progress = (unsigned*)(tb + key_bytes * 2 * (pairs ? 2 : 1));

  // every merge pass in one persistent launch (the window kernel; per-CTA
  // progress flags instead of pass boundaries), unless a pass needs another
  // kernel: pairs whose final key / value outputs differ in 16-byte phase
  // take the plain kernel for the last pass
  const bool last_phase_ok = !pairs || (((uintptr_t)out_k ^ (uintptr_t)out_v) & 15) == 0;
  const bool multi = P >= 2 && use_tma && var.merge_multi && last_phase_ok && !multipass_disabled() &&
                     !trace_requested();
  // the block sort zeroes the progress flags (no memset between the two launches)
  SortArgs sa{in_k, in_v, P == 0 ? out_k : X, P == 0 ? out_v : XV, (long long)n, f32 ? 1 : 0,
              (f32 && P == 0) ? 1 : 0, cf ? 1 : 0, multi ? progress : nullptr, multi ? MAX_PROGRESS_CTAS : 0};
  long long grid_bs = tiles_bs;
  if (one_sm && tiles_bs > sm_count()) {
    grid_bs = sm_count();
    sa.ntiles = tiles_bs;
  }
  cudaError_t e = launch("block_sort", n, s, [&] {
    return bs2 ? vbs.block_sort2(sa, grid_bs, s) : vbs.block_sort(sa, grid_bs, s);
  });
  if (e != cudaSuccess) return cuda_fail(e);
  if (multi) {
    MergeArgs ma{X, XV, out_k, out_v, (long long)n, Tbs, 1 + lg_bs, f32 ? 1 : 0, cf ? 1 : 0, nullptr, 0, nullptr};
    ma.npass = P;
    ma.progress = progress;
    ma.buf_k[0] = X;
    ma.buf_k[1] = Y;
    ma.buf_v[0] = XV;
    ma.buf_v[1] = YV;
    ma.trace = multi_trace();
    e = launch("merge_passes", n * (uint64_t)P, s, [&] { return var.merge_multi(ma, tiles, s); });
    return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
  }
  for (int i = 1; i <= P; ++i) {
    uint32_t* sk = (i & 1) ? X : Y;
    uint32_t* sv = (i & 1) ? XV : YV;
    uint32_t* dk = i == P ? out_k : ((i & 1) ? Y : X);
    uint32_t* dv = i == P ? out_v : ((i & 1) ? YV : XV);
    MergeArgs ma{sk, sv, dk, dv, (long long)n, Tbs << (i - 1), i + lg_bs,
                 (f32 && i == P) ? 1 : 0, cf ? 1 : 0, nullptr, 0, trace_for_pass(i)};
    // the persistent kernels bulk-store keys and values at one 16-byte phase
    // (the keys'): a final pass into key / value outputs of different phases
    // takes the plain kernel
    const bool phase_ok = !pairs || i < P || (((uintptr_t)out_k ^ (uintptr_t)out_v) & 15) == 0;
    long long grid = tiles;
    if (one_sm && tiles > sm_count()) {
      grid = sm_count();
      ma.ntiles = tiles;
    }
    if (use_tma && phase_ok)
      e = launch("merge_pass", n, s, [&] { return var.merge_tma(ma, tiles, s); });
    else
      e = launch("merge_pass", n, s, [&] { return var.merge(ma, grid, s); });
    if (e != cudaSuccess) return cuda_fail(e);
  }
  return BCF_SUCCESS;
}

// ---------------------------------------------------------------------------
// host-buffer batches: H2D of batch i+1 and D2H of batch i-1 overlap the sort
// of batch i (copy engines run both directions at once); two device slots
// ---------------------------------------------------------------------------
struct CopyStreams {
  cudaStream_t h2d = nullptr, d2h = nullptr;
};

static cudaError_t copy_streams(CopyStreams& cs) {
  static std::mutex mu;
  static CopyStreams per_dev[64];
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(mu);
  CopyStreams& c = per_dev[dev];
  if (!c.h2d) {
    e = cudaStreamCreateWithFlags(&c.h2d, cudaStreamNonBlocking);
    if (e != cudaSuccess) return e;
    e = cudaStreamCreateWithFlags(&c.d2h, cudaStreamNonBlocking);
    if (e != cudaSuccess) return e;
  }
  cs = c;
  return cudaSuccess;
}

static bcf_status host_batch_impl(const uint32_t* const* h_in, uint32_t* const* h_out, int32_t nbatch,
                                  uint64_t n, void* d_temp, size_t* temp_bytes, const bcf_params* pp,
                                  cudaStream_t s, bool f32) {
  if (!temp_bytes || nbatch < 0) return BCF_ERROR_INVALID_VALUE;
  size_t sort_bytes = 0;
  bcf_status st = sort_impl(nullptr, nullptr, nullptr, nullptr, n, nullptr, &sort_bytes, pp, s, f32, false);
  if (st != BCF_SUCCESS) return st;
  const size_t key_bytes = align_up((size_t)n * sizeof(uint32_t), 256);
  const size_t need = 256 + 4 * key_bytes + sort_bytes;
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return BCF_SUCCESS;
  }
  if (*temp_bytes < need) return BCF_ERROR_TEMP_TOO_SMALL;
  if (nbatch == 0 || n == 0) return BCF_SUCCESS;
  if (!h_in || !h_out) return BCF_ERROR_INVALID_VALUE;
  for (int i = 0; i < nbatch; ++i)
    if (!h_in[i] || !h_out[i]) return BCF_ERROR_INVALID_VALUE;
  CopyStreams cs;
  cudaError_t e = copy_streams(cs);
  if (e != cudaSuccess) return cuda_fail(e);
  char* tb = (char*)align_up((size_t)d_temp, 256);
  uint32_t* din[2] = {(uint32_t*)tb, (uint32_t*)(tb + key_bytes)};
  uint32_t* dout[2] = {(uint32_t*)(tb + 2 * key_bytes), (uint32_t*)(tb + 3 * key_bytes)};
  void* stemp = tb + 4 * key_bytes;
  // events: entry (caller-stream order), per slot: input landed, sorted, output read back
  cudaEvent_t ev[7];
  for (auto& x : ev) {
    e = cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(e);
  }
  cudaEvent_t entry = ev[0], in_ok[2] = {ev[1], ev[2]}, sorted[2] = {ev[3], ev[4]}, out_ok[2] = {ev[5], ev[6]};
  auto chk = [&](cudaError_t x) {
    if (x != cudaSuccess && e == cudaSuccess) e = x;
  };
  chk(cudaEventRecord(entry, s));
  chk(cudaStreamWaitEvent(cs.h2d, entry, 0));
  chk(cudaStreamWaitEvent(cs.d2h, entry, 0));
  const size_t bytes = (size_t)n * sizeof(uint32_t);
  for (int i = 0; i < nbatch && e == cudaSuccess; ++i) {
    const int k = i & 1;
    if (i >= 2) chk(cudaStreamWaitEvent(cs.h2d, sorted[k], 0));  // sort i-2 has read din[k]
    chk(cudaMemcpyAsync(din[k], h_in[i], bytes, cudaMemcpyHostToDevice, cs.h2d));
    chk(cudaEventRecord(in_ok[k], cs.h2d));
    chk(cudaStreamWaitEvent(s, in_ok[k], 0));
    if (i >= 2) chk(cudaStreamWaitEvent(s, out_ok[k], 0));  // D2H i-2 has read dout[k]
    if (e != cudaSuccess) break;
    size_t sb = sort_bytes;
    st = sort_impl(din[k], dout[k], nullptr, nullptr, n, stemp, &sb, pp, s, f32, false);
    if (st != BCF_SUCCESS) break;
    chk(cudaEventRecord(sorted[k], s));
    chk(cudaStreamWaitEvent(cs.d2h, sorted[k], 0));
    chk(cudaMemcpyAsync(h_out[i], dout[k], bytes, cudaMemcpyDeviceToHost, cs.d2h));
    chk(cudaEventRecord(out_ok[k], cs.d2h));
  }
  // the caller's stream completes after the last read-back
  chk(cudaEventRecord(out_ok[0], cs.d2h));
  chk(cudaStreamWaitEvent(s, out_ok[0], 0));
  chk(cudaStreamWaitEvent(cs.h2d, out_ok[0], 0));
  for (auto& x : ev) cudaEventDestroy(x);
  if (st != BCF_SUCCESS) return st;
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

// ---------------------------------------------------------------------------
// distributed helpers
// ---------------------------------------------------------------------------
__global__ void split_counts_kernel(const uint32_t* __restrict__ a, unsigned long long n,
                                    const uint32_t* __restrict__ piv, int npiv,
                                    unsigned long long* __restrict__ lt, unsigned long long* __restrict__ le) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= npiv) return;
  const uint32_t v = piv[i];
  unsigned long long lo = 0, hi = n;  // first index with a[idx] >= v
  while (lo < hi) {
    const unsigned long long mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1; else hi = mid;
  }
  lt[i] = lo;
  hi = n;  // first index with a[idx] > v
  while (lo < hi) {
    const unsigned long long mid = (lo + hi) >> 1;
    if (a[mid] <= v) lo = mid + 1; else hi = mid;
  }
  le[i] = lo;
}

}  // namespace bcf

using namespace bcf;

extern "C" {

void bcf_default_params(bcf_params* p) {
  if (!p) return;
  p->items_per_thread = DEFAULT_E;
  p->block_threads = DEFAULT_U;
  p->algo = BCF_ALGO_CONFLICT_FREE;
}

void bcf_default_pairs_params(bcf_params* p) {
  if (!p) return;
  p->items_per_thread = DEFAULT_E_PAIRS;
  p->block_threads = DEFAULT_U_PAIRS;
  p->algo = BCF_ALGO_CONFLICT_FREE;
}

bcf_status bcf_sort_u32(const uint32_t* d_in, uint32_t* d_out, uint64_t n, void* d_temp,
                        size_t* temp_bytes, const bcf_params* p, void* stream) {
  return sort_impl(d_in, d_out, nullptr, nullptr, n, d_temp, temp_bytes, p, (cudaStream_t)stream, false,
                   false);
}

bcf_status bcf_sort_f32(const float* d_in, float* d_out, uint64_t n, void* d_temp, size_t* temp_bytes,
                        const bcf_params* p, void* stream) {
  return sort_impl((const uint32_t*)d_in, (uint32_t*)d_out, nullptr, nullptr, n, d_temp, temp_bytes, p,
                   (cudaStream_t)stream, true, false);
}

bcf_status bcf_sort_plan(uint64_t n, const bcf_params* pp, int32_t pairs, int64_t* block_sort_tile,
                         int64_t* merge_tile, int32_t* merge_passes) {
  Params p;
  bcf_status st = resolve(pp, p, pairs != 0);
  if (st != BCF_SUCCESS) return st;
  const bool cf = p.algo == BCF_ALGO_CONFLICT_FREE;
  const int Ubs = bs_threads(p, cf, pairs != 0);
  const long long Tbs = (long long)Ubs * p.E * (!one_cta_per_sm() && use_bs2(p, cf, pairs != 0, Ubs) ? 2 : 1);
  int P = 0;
  while ((Tbs << P) < (long long)n) ++P;
  if (block_sort_tile) *block_sort_tile = Tbs;
  if (merge_tile) *merge_tile = (long long)p.U * p.E;
  if (merge_passes) *merge_passes = P;
  return BCF_SUCCESS;
}

bcf_status bcf_sort_u32_host_batch(const uint32_t* const* h_in, uint32_t* const* h_out, int32_t nbatch,
                                   uint64_t n, void* d_temp, size_t* temp_bytes, const bcf_params* p,
                                   void* stream) {
  return host_batch_impl(h_in, h_out, nbatch, n, d_temp, temp_bytes, p, (cudaStream_t)stream, false);
}

bcf_status bcf_sort_pairs_u32(const uint32_t* d_keys_in, uint32_t* d_keys_out, const uint32_t* d_vals_in,
                              uint32_t* d_vals_out, uint64_t n, void* d_temp, size_t* temp_bytes,
                              const bcf_params* p, void* stream) {
  return sort_impl(d_keys_in, d_keys_out, d_vals_in, d_vals_out, n, d_temp, temp_bytes, p,
                   (cudaStream_t)stream, false, true);
}

static bool worst_case_params_ok(uint64_t n, int32_t E, int32_t u) {
  // merge levels R = E * 2^e need u a power of two; the closed form's small
  // divisions are exact below 2^40 keys
  return E >= 2 && E <= 32 && u >= 32 && (u & (u - 1)) == 0 && n <= (1ull << 36);
}

bcf_status bcf_worst_case_u32_host(uint32_t* h_out, uint64_t n, int32_t E, int32_t u, uint64_t seed) {
  if (n > 0 && !h_out) return BCF_ERROR_INVALID_VALUE;
  if (!worst_case_params_ok(n, E, u)) return BCF_ERROR_UNSUPPORTED;
  return wc::generate_host(h_out, n, E, u, seed) ? BCF_SUCCESS : BCF_ERROR_UNSUPPORTED;
}

bcf_status bcf_worst_case_u32(uint32_t* d_out, uint64_t n, int32_t E, int32_t u, uint64_t seed,
                              void* stream) {
  if (n > 0 && !d_out) return BCF_ERROR_INVALID_VALUE;
  if (!worst_case_params_ok(n, E, u)) return BCF_ERROR_UNSUPPORTED;
  if (n == 0) return BCF_SUCCESS;
  bool ok = true;
  cudaError_t e = launch("worst_case", n, (cudaStream_t)stream, [&] {
    return wc::generate_device(d_out, n, E, u, seed, (cudaStream_t)stream, &ok);
  });
  if (e != cudaSuccess) return cuda_fail(e);
  return ok ? BCF_SUCCESS : BCF_ERROR_UNSUPPORTED;
}

bcf_status bcf_split_counts_u32(const uint32_t* d_sorted, uint64_t n, const uint32_t* d_pivots, int32_t npiv,
                                uint64_t* d_lt_counts, uint64_t* d_le_counts, void* stream) {
  if (npiv < 0) return BCF_ERROR_INVALID_VALUE;
  if (npiv == 0) return BCF_SUCCESS;
  if ((n > 0 && !d_sorted) || !d_pivots || !d_lt_counts || !d_le_counts) return BCF_ERROR_INVALID_VALUE;
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = launch("split_counts", (uint64_t)npiv, s, [&] {
    split_counts_kernel<<<(npiv + 127) / 128, 128, 0, s>>>(d_sorted, (unsigned long long)n, d_pivots, npiv,
                                                          (unsigned long long*)d_lt_counts,
                                                          (unsigned long long*)d_le_counts);
    return cudaGetLastError();
  });
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

// the one group descriptor of bcf_merge_u32, written by a 1-thread kernel
// (a kernel parameter, not a pageable H2D copy: the call stays capturable
// into a CUDA graph)
__global__ void write_desc_kernel(GroupDesc* d, GroupDesc g) { *d = g; }

// bcf_merge_runs_u32's per-pass descriptor tables, likewise written from
// kernel parameters (chunks of DESC_CHUNK descriptors, one thread each)
constexpr int DESC_CHUNK = 24;
struct DescChunk {
  GroupDesc g[DESC_CHUNK];
  int count;
};
__global__ void write_table_kernel(GroupDesc* d, DescChunk c) {
  if ((int)threadIdx.x < c.count) d[threadIdx.x] = c.g[threadIdx.x];
}
static cudaError_t write_table(GroupDesc* d, const std::vector<GroupDesc>& tab, cudaStream_t s) {
  for (size_t i = 0; i < tab.size(); i += DESC_CHUNK) {
    DescChunk c;
    c.count = (int)std::min<size_t>(DESC_CHUNK, tab.size() - i);
    for (int j = 0; j < c.count; ++j) c.g[j] = tab[i + j];
    write_table_kernel<<<1, DESC_CHUNK, 0, s>>>(d + i, c);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// B reversed into temp for the window kernel, whose bulk copies need B
// stored descending (element y of B at out[nb-1-y])
__global__ void reverse_u32_kernel(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, long long n) {
  for (long long j = blockIdx.x * (long long)blockDim.x + threadIdx.x; j < n; j += (long long)gridDim.x * blockDim.x)
    out[j] = __ldg(in + (n - 1 - j));
}

// run_ptrs (host array of nruns device pointers, keys only): run r is read
// from run_ptrs[r] (local or peer-mapped memory) instead of d_runs + offset;
// pass 1 then reads every run through its own pointer (the plain kernel's
// GroupDesc a_ptr / b_ptr), later passes are local
static bcf_status merge_runs_impl(const uint32_t* d_runs, const uint32_t* const* run_ptrs, const uint32_t* d_run_vals,
                                  const uint64_t* h_run_offsets, int32_t nruns, uint32_t* d_out, uint32_t* d_out_vals,
                                  void* d_temp, size_t* temp_bytes, const bcf_params* pp, void* stream) {
  // Pairwise merge tree over the runs in run order (run 2g is A, 2g+1 is B,
  // ties to A = the lower run).  Pass 1 reads the caller's ascending runs with
  // the plain table-mode kernel; it and every later non-final pass write odd
  // groups DESCENDING (the sort's CF run directions), each output run at its
  // own position in a temp buffer with 4 words of gap, a descending run
  // shifted so that b_off = a_off - nb (mod 4) against its A partner.  Passes
  // >= 2 then run on the persistent TMA/window kernels exactly like the
  // sort's passes (B bulk-copied straight into its reversed slot).
  if (!temp_bytes || nruns < 0 || (nruns > 0 && !h_run_offsets)) return BCF_ERROR_INVALID_VALUE;
  const bool pairs = d_run_vals != nullptr;
  Params p;
  bcf_status st = resolve(pp, p, pairs);
  if (st != BCF_SUCCESS) return st;
  if (p.algo != BCF_ALGO_CONFLICT_FREE) return BCF_ERROR_UNSUPPORTED;
  const uint64_t n = nruns > 0 ? h_run_offsets[nruns] : 0;
  for (int r = 0; r < nruns; ++r)
    if (h_run_offsets[r + 1] < h_run_offsets[r] || h_run_offsets[0] != 0) return BCF_ERROR_INVALID_VALUE;
  // per output run: up to 3 phase words + 4 words of gap; per reversed B run
  // before pass 1: up to 3 phase words + 8 words of gap
  const size_t buf_words = (size_t)n + 12 * ((size_t)nruns + 2) + 64;
  const size_t key_bytes = align_up(buf_words * sizeof(uint32_t), 256);
  const size_t table_bytes = align_up(sizeof(GroupDesc) * (size_t)(nruns / 2 + 1), 256);
  // + one buffer (per array) for the odd runs reversed before pass 1
  const size_t need = 256 + key_bytes * 3 * (pairs ? 2 : 1) + table_bytes * 64;
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return BCF_SUCCESS;
  }
  if (*temp_bytes < need) return BCF_ERROR_TEMP_TOO_SMALL;
  if (n == 0) return BCF_SUCCESS;
  if ((!d_runs && !run_ptrs) || !d_out || (pairs && (!d_out_vals || run_ptrs))) return BCF_ERROR_INVALID_VALUE;
  if (run_ptrs)
    for (int r = 0; r < nruns; ++r)
      if (!run_ptrs[r] && h_run_offsets[r + 1] > h_run_offsets[r]) return BCF_ERROR_INVALID_VALUE;
  cudaStream_t s = (cudaStream_t)stream;
  if (nruns == 1) {
    cudaError_t e = cudaMemcpyAsync(d_out, run_ptrs ? run_ptrs[0] : d_runs, n * 4, cudaMemcpyDeviceToDevice, s);
    if (e == cudaSuccess && pairs) e = cudaMemcpyAsync(d_out_vals, d_run_vals, n * 4, cudaMemcpyDeviceToDevice, s);
    return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
  }
  const Variant& var = launch_table().v[p.E][u_index(p.U)][0][pairs ? 1 : 0];
  if (!var.merge_table || !var.merge) return BCF_ERROR_UNSUPPORTED;
  const bool use_tma = var.merge_tma != nullptr && !tma_disabled();
  const long long T = (long long)p.U * p.E;
  char* tb = (char*)align_up((size_t)d_temp, 256);
  uint32_t* tk[2] = {(uint32_t*)tb, (uint32_t*)(tb + key_bytes)};
  uint32_t* tv[2] = {pairs ? (uint32_t*)(tb + 2 * key_bytes) : nullptr,
                     pairs ? (uint32_t*)(tb + 3 * key_bytes) : nullptr};
  uint32_t* rk = (uint32_t*)(tb + key_bytes * (pairs ? 4 : 2));  // reversed odd runs
  uint32_t* rv = pairs ? (uint32_t*)(tb + key_bytes * 5) : nullptr;
  GroupDesc* dtab = (GroupDesc*)(tb + key_bytes * 3 * (pairs ? 2 : 1));
  int P = 0;
  while ((1 << P) < nruns) ++P;
  struct Run {
    long long pos, len;
    int desc;
  };
  std::vector<Run> runs(nruns);
  for (int r = 0; r < nruns; ++r)
    runs[r] = {(long long)h_run_offsets[r], (long long)(h_run_offsets[r + 1] - h_run_offsets[r]), 0};
  // Pass 1 on the window kernel too: the odd (B) runs reversed into rk
  // (+8 B per B key), each at word phase A pos - len (mod 4) against its A
  // partner, read through src_kb / src_vb; A straight from the caller's
  // 16-byte aligned runs.  Bounded run count (one reverse launch per B run).
  const bool rev1 = !run_ptrs && var.merge_win != nullptr && !tma_disabled() && nruns <= 64 &&
                    ((uintptr_t)d_runs & 15) == 0 &&
                    (!pairs || (((uintptr_t)d_run_vals & 15) == 0 &&
                                (P > 1 || (((uintptr_t)d_out ^ (uintptr_t)d_out_vals) & 15) == 0)));
  if (rev1) {
    long long cur = 0;
    for (int r = 1; r < nruns; r += 2) {
      const long long len = runs[r].len;
      const long long pos = cur + ((((runs[r - 1].pos - len - cur) % 4) + 4) % 4);
      cur = pos + len + 8;
      runs[r] = {pos, len, 1};
      if (len == 0) continue;
      const long long src0 = (long long)h_run_offsets[r];
      const long long blocks = std::min<long long>((len + 255) / 256, 148LL * 16);
      cudaError_t e = launch("merge_reverse", (uint64_t)len, s, [&] {
        reverse_u32_kernel<<<(unsigned)blocks, 256, 0, s>>>(d_runs + src0, rk + pos, len);
        if (pairs) reverse_u32_kernel<<<(unsigned)blocks, 256, 0, s>>>(d_run_vals + src0, rv + pos, len);
        return cudaGetLastError();
      });
      if (e != cudaSuccess) return cuda_fail(e);
    }
  }
  const uint32_t* srck = d_runs;
  const uint32_t* srcv = d_run_vals;
  for (int i = 1; i <= P; ++i) {
    const bool last = i == P;
    uint32_t* dk = last ? d_out : tk[i & 1];
    uint32_t* dv = last ? d_out_vals : tv[i & 1];
    std::vector<GroupDesc> tab;
    std::vector<Run> next;
    long long tiles = 0, cursor = 0;
    const int nr = (int)runs.size();
    for (int r = 0, g = 0; r < nr; r += 2, ++g) {
      const Run& A = runs[r];
      const Run B = r + 1 < nr ? runs[r + 1] : Run{A.pos + A.len, 0, 1};
      GroupDesc gd{};
      gd.a_off = A.pos;
      gd.na = A.len;
      gd.b_off = B.pos;
      gd.nb = B.len;
      gd.b_desc = B.desc;
      if (i == 1 && run_ptrs) {  // the caller's runs, each through its own pointer
        gd.a_ptr = run_ptrs[r];
        gd.b_ptr = r + 1 < nr ? run_ptrs[r + 1] : run_ptrs[r];
        gd.a_off = 0;
        gd.b_off = 0;
      }
      Run o{0, A.len + B.len, 0};
      if (!last) {
        o.desc = g & 1;
        o.pos = cursor;
        // a descending output (next pass's B) sits at pos = A' pos - len (mod 4)
        // against its partner A' = the previous group's output
        if (o.desc) o.pos += (((next.back().pos - o.len - cursor) % 4) + 4) % 4;
        cursor = o.pos + o.len + 4;
      }
      gd.out_off = o.pos;
      gd.out_desc = o.desc;
      gd.tile_begin = tiles;
      tiles += (o.len + T - 1) / T;
      if (o.len > 0) tab.push_back(gd);
      next.push_back(o);
    }
    GroupDesc* dt = dtab + (size_t)(i - 1) * (table_bytes / sizeof(GroupDesc));
    cudaError_t e = write_table(dt, tab, s);  // kernel launches: capturable into a CUDA graph
    if (e != cudaSuccess) return cuda_fail(e);
    MergeArgs ma{srck, srcv, dk, dv, (long long)n, 0, 0, 0, 0, dt, (int)tab.size(), nullptr};
    if (i == 1 && rev1) {
      ma.src_kb = rk;
      ma.src_vb = rv;
      e = launch("merge_runs", n, s, [&] { return var.merge_win(ma, tiles, s); });
    } else if (i == 1)  // the caller's runs: all ascending
      e = launch("merge_runs", n, s, [&] { return var.merge_table(ma, tiles, s); });
    else if (use_tma && (!pairs || !last || (((uintptr_t)d_out ^ (uintptr_t)d_out_vals) & 15) == 0))
      e = launch("merge_runs", n, s, [&] { return var.merge_tma(ma, tiles, s); });
    else
      e = launch("merge_runs", n, s, [&] { return var.merge(ma, tiles, s); });
    if (e != cudaSuccess) return cuda_fail(e);
    srck = dk;
    srcv = dv;
    runs.swap(next);
  }
  return BCF_SUCCESS;
}

bcf_status bcf_merge_u32(const uint32_t* d_a, uint64_t na, const uint32_t* d_b, uint64_t nb,
                         const uint32_t* d_a_vals, const uint32_t* d_b_vals, uint32_t* d_out,
                         uint32_t* d_out_vals, void* d_temp, size_t* temp_bytes, const bcf_params* pp,
                         void* stream) {
  // One CF merge pass (table mode, one group) with B read from its own base
  // pointer: the merge step of the paper's pairwise mergesort exposed as a
  // primitive (PAPER.md:59-61 merge path; :380 "any parallel scan of a pair
  // of arrays").  Ties go to A.
  if (!temp_bytes) return BCF_ERROR_INVALID_VALUE;
  const bool pairs = d_a_vals != nullptr || d_b_vals != nullptr || d_out_vals != nullptr;
  Params p;
  bcf_status st = resolve(pp, p, pairs);
  if (st != BCF_SUCCESS) return st;
  if (p.algo != BCF_ALGO_CONFLICT_FREE) return BCF_ERROR_UNSUPPORTED;
  // keys only: room for B reversed (window kernel path), +8 words of phase/tail slack
  const size_t need = 256 + align_up(sizeof(GroupDesc), 256) + align_up(4 * ((size_t)nb + 8), 256) * (pairs ? 2 : 1);
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return BCF_SUCCESS;
  }
  if (*temp_bytes < need) return BCF_ERROR_TEMP_TOO_SMALL;
  const uint64_t n = na + nb;
  if (n == 0) return BCF_SUCCESS;
  if ((na && !d_a) || (nb && !d_b) || !d_out) return BCF_ERROR_INVALID_VALUE;
  if (pairs && ((na && !d_a_vals) || (nb && !d_b_vals) || !d_out_vals)) return BCF_ERROR_INVALID_VALUE;
  cudaStream_t s = (cudaStream_t)stream;
  if (na == 0 || nb == 0) {  // one side empty: the merge is a copy
    const uint32_t* k = na ? d_a : d_b;
    const uint32_t* v = na ? d_a_vals : d_b_vals;
    cudaError_t e = cudaMemcpyAsync(d_out, k, n * 4, cudaMemcpyDeviceToDevice, s);
    if (e == cudaSuccess && pairs) e = cudaMemcpyAsync(d_out_vals, v, n * 4, cudaMemcpyDeviceToDevice, s);
    return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
  }
  const Variant& var = launch_table().v[p.E][u_index(p.U)][0][pairs ? 1 : 0];
  if (!var.merge_table) return BCF_ERROR_UNSUPPORTED;
  const long long T = (long long)p.U * p.E;
  const long long tiles = (long long)((n + T - 1) / T);
  GroupDesc g{};
  g.na = (long long)na;
  g.nb = (long long)nb;
  GroupDesc* dt = (GroupDesc*)align_up((size_t)d_temp, 256);
  const bool win_ok = var.merge_win && ((uintptr_t)d_a & 15) == 0 && !tma_disabled() &&
                      (!pairs || (((uintptr_t)d_a_vals & 15) == 0 && (((uintptr_t)d_out ^ (uintptr_t)d_out_vals) & 15) == 0));
  if (win_ok) {
    // persistent window kernel (0.8 of HBM per pass at 2^28): B reversed into
    // temp at word phase b_off = -nb mod 4, so that A's and B's windows share
    // one 16-byte phase (a_off - b_off - nb = 0 mod 4, as in the sort's passes)
    uint32_t* rb = (uint32_t*)((char*)dt + align_up(sizeof(GroupDesc), 256));
    g.b_off = (long long)((4 - (nb & 3)) & 3);
    g.b_desc = 1;
    write_desc_kernel<<<1, 1, 0, s>>>(dt, g);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e);
    const long long blocks = std::min<long long>((long long)((nb + 255) / 256), 148LL * 16);
    e = launch("merge_reverse", nb, s, [&] {
      reverse_u32_kernel<<<(unsigned)blocks, 256, 0, s>>>(d_b, rb + g.b_off, (long long)nb);
      return cudaGetLastError();
    });
    if (e != cudaSuccess) return cuda_fail(e);
    uint32_t* rbv = pairs ? rb + align_up(4 * ((size_t)nb + 8), 256) / 4 : nullptr;
    if (pairs) {
      e = launch("merge_reverse", nb, s, [&] {
        reverse_u32_kernel<<<(unsigned)blocks, 256, 0, s>>>(d_b_vals, rbv + g.b_off, (long long)nb);
        return cudaGetLastError();
      });
      if (e != cudaSuccess) return cuda_fail(e);
    }
    MergeArgs ma{d_a, d_a_vals, d_out, d_out_vals, (long long)n, 0, 0, 0, 0, dt, 1, nullptr, rb, rbv};
    e = launch("merge", n, s, [&] { return var.merge_win(ma, tiles, s); });
    return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
  }
  write_desc_kernel<<<1, 1, 0, s>>>(dt, g);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e);
  MergeArgs ma{d_a, d_a_vals, d_out, d_out_vals, (long long)n, 0, 0, 0, 0, dt, 1, nullptr, d_b, d_b_vals};
  e = launch("merge", n, s, [&] { return var.merge_table(ma, tiles, s); });
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

bcf_status bcf_set_op_u32(int32_t op, const uint32_t* d_a, uint64_t na, const uint32_t* d_b, uint64_t nb,
                          uint32_t* d_out, uint32_t* d_out_src, uint64_t* d_count, void* d_temp, size_t* temp_bytes,
                          const bcf_params* pp, void* stream) {
  if (!temp_bytes || op < BCF_SET_UNION || op > BCF_SET_SYMMETRIC_DIFFERENCE) return BCF_ERROR_INVALID_VALUE;
  if (na >= (1ull << 31) || nb >= (1ull << 31)) return BCF_ERROR_UNSUPPORTED;  // 31-bit source indices
  const uint64_t n = na + nb;
  // merge temp (pairs: keys + source tags)
  size_t mtb = 0;
  bcf_status st = bcf_merge_u32(nullptr, na, nullptr, nb, (const uint32_t*)16, (const uint32_t*)16, nullptr,
                                (uint32_t*)16, nullptr, &mtb, pp, stream);
  if (st != BCF_SUCCESS) return st;
  const size_t ta_b = align_up(na * 4 + 4, 256), tb_b = align_up(nb * 4 + 4, 256), m_b = align_up(n * 4 + 4, 256);
  const size_t c_b = align_up(((size_t)setops::compact_blocks((long long)n) + 1) * 8, 256);
  const size_t need = 256 + ta_b + tb_b + 2 * m_b + c_b + mtb;
  if (d_temp == nullptr) {
    *temp_bytes = need;
    return BCF_SUCCESS;
  }
  if (*temp_bytes < need) return BCF_ERROR_TEMP_TOO_SMALL;
  if (!d_count || (n > 0 && !d_out) || (na && !d_a) || (nb && !d_b)) return BCF_ERROR_INVALID_VALUE;
  cudaStream_t s = (cudaStream_t)stream;
  char* tb = (char*)align_up((size_t)d_temp, 256);
  uint32_t* ta = (uint32_t*)tb;
  uint32_t* tbt = (uint32_t*)(tb + ta_b);
  uint32_t* M = (uint32_t*)(tb + ta_b + tb_b);
  uint32_t* V = (uint32_t*)(tb + ta_b + tb_b + m_b);
  unsigned long long* counts = (unsigned long long*)(tb + ta_b + tb_b + 2 * m_b);
  void* mt = tb + ta_b + tb_b + 2 * m_b + c_b;
  cudaError_t e = launch("setop_tags", n, s, [&] { return setops::make_tags(ta, (long long)na, tbt, (long long)nb, s); });
  if (e != cudaSuccess) return cuda_fail(e);
  if (n > 0) {
    size_t m2 = mtb;
    st = bcf_merge_u32(d_a, na, d_b, nb, na ? ta : nullptr, nb ? tbt : nullptr, M, V, mt, &m2, pp, stream);
    if (st != BCF_SUCCESS) return st;
  }
  e = launch("setop_compact", n, s, [&] {
    return setops::compact(op, M, V, (long long)n, counts, (unsigned long long*)d_count, d_out, d_out_src, s);
  });
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

bcf_status bcf_merge_runs_u32(const uint32_t* d_runs, const uint32_t* d_run_vals, const uint64_t* h_run_offsets,
                              int32_t nruns, uint32_t* d_out, uint32_t* d_out_vals, void* d_temp,
                              size_t* temp_bytes, const bcf_params* pp, void* stream) {
  return merge_runs_impl(d_runs, nullptr, d_run_vals, h_run_offsets, nruns, d_out, d_out_vals, d_temp, temp_bytes,
                         pp, stream);
}

bcf_status bcf_merge_runs_ptrs_u32(const uint32_t* const* h_run_ptrs, const uint64_t* h_run_lens, int32_t nruns,
                                   uint32_t* d_out, void* d_temp, size_t* temp_bytes, const bcf_params* pp,
                                   void* stream) {
  if (nruns < 0 || (nruns > 0 && (!h_run_ptrs || !h_run_lens))) return BCF_ERROR_INVALID_VALUE;
  if (nruns > 4096) return BCF_ERROR_UNSUPPORTED;
  uint64_t offs[4097];
  offs[0] = 0;
  for (int r = 0; r < nruns; ++r) offs[r + 1] = offs[r] + h_run_lens[r];
  return merge_runs_impl(nullptr, d_temp ? h_run_ptrs : (const uint32_t* const*)nullptr, nullptr, offs, nruns, d_out,
                         nullptr, d_temp, temp_bytes, pp, stream);
}

// ---- CUDA IPC (one node, one process per GPU; bcf_merge_runs_ptrs_u32) ----
typedef int (*cuMemGetAddressRange_t)(unsigned long long*, size_t*, unsigned long long);
static cuMemGetAddressRange_t address_range_fn() {
  static cuMemGetAddressRange_t fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      f = nullptr;
    return (cuMemGetAddressRange_t)f;
  }();
  return fn;
}

bcf_status bcf_ipc_export(const void* d_ptr, void* handle, uint64_t* offset) {
  if (!d_ptr || !handle || !offset) return BCF_ERROR_INVALID_VALUE;
  cuMemGetAddressRange_t range = address_range_fn();
  if (!range) return BCF_ERROR_UNSUPPORTED;
  unsigned long long base = 0;
  size_t size = 0;
  if (range(&base, &size, (unsigned long long)(uintptr_t)d_ptr) != 0) return BCF_ERROR_INVALID_VALUE;
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaIpcGetMemHandle(&h, (void*)(uintptr_t)base);
  if (e != cudaSuccess) return cuda_fail(e);
  std::memcpy(handle, &h, sizeof(h));
  *offset = (uint64_t)((uintptr_t)d_ptr - (uintptr_t)base);
  return BCF_SUCCESS;
}

bcf_status bcf_ipc_open(const void* handle, void** d_base) {
  if (!handle || !d_base) return BCF_ERROR_INVALID_VALUE;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  cudaError_t e = cudaIpcOpenMemHandle(d_base, h, cudaIpcMemLazyEnablePeerAccess);
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

bcf_status bcf_ipc_close(void* d_base) {
  if (!d_base) return BCF_ERROR_INVALID_VALUE;
  cudaError_t e = cudaIpcCloseMemHandle(d_base);
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

const char* bcf_status_string(bcf_status s) {
  switch (s) {
    case BCF_SUCCESS: return "BCF_SUCCESS";
    case BCF_ERROR_INVALID_VALUE: return "BCF_ERROR_INVALID_VALUE";
    case BCF_ERROR_UNSUPPORTED: return "BCF_ERROR_UNSUPPORTED";
    case BCF_ERROR_CUDA: return "BCF_ERROR_CUDA";
    case BCF_ERROR_TEMP_TOO_SMALL: return "BCF_ERROR_TEMP_TOO_SMALL";
  }
  return "BCF_ERROR_UNKNOWN";
}

int32_t bcf_abi_version(void) { return BCF_ABI_VERSION; }
int32_t bcf_last_cuda_error(void) { return t_last_cuda_error; }

bcf_status bcf_profile_enable(int32_t on) {
  g_prof_on.store(on ? 1 : 0);
  return BCF_SUCCESS;
}

bcf_status bcf_profile_collect(bcf_kernel_stats* out, int32_t max, int32_t* count) {
  std::lock_guard<std::mutex> lk(g_prof_mu);
  std::vector<bcf_kernel_stats> acc;
  cudaError_t err = cudaSuccess;
  for (auto& r : g_recs) {
    float ms = 0.f;
    cudaError_t e = cudaEventSynchronize(r.b);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, r.a, r.b);
    if (e != cudaSuccess) err = e;
    auto it = std::find_if(acc.begin(), acc.end(), [&](const bcf_kernel_stats& k) { return std::strcmp(k.name, r.name) == 0; });
    if (it == acc.end()) {
      bcf_kernel_stats k{};
      std::strncpy(k.name, r.name, sizeof(k.name) - 1);
      acc.push_back(k);
      it = acc.end() - 1;
    }
    it->launches += 1;
    it->total_ms += ms;
    it->keys += r.keys;
    g_pool.push_back(r.a);
    g_pool.push_back(r.b);
  }
  g_recs.clear();
  if (count) *count = (int32_t)acc.size();
  for (int i = 0; i < (int)acc.size() && i < max && out; ++i) out[i] = acc[i];
  return err == cudaSuccess ? BCF_SUCCESS : cuda_fail(err);
}

int64_t bcf_launch_count(void) { return g_launches.load(); }

bcf_status bcf_debug_trace_copy(void* host, uint64_t bytes) {
  if (!g_trace) return BCF_ERROR_INVALID_VALUE;
  if (bytes > TRACE_WORDS * 8) bytes = TRACE_WORDS * 8;
  cudaError_t e = cudaMemcpy(host, g_trace, bytes, cudaMemcpyDeviceToHost);
  return e == cudaSuccess ? BCF_SUCCESS : cuda_fail(e);
}

}  // extern "C"
