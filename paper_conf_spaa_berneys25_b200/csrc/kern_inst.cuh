// kern_inst.cuh -- explicit instantiation of the kernels for one E and the
// three block sizes; included by kern_E<E>.cu with BCF_E defined.
#pragma once
#include <cstdlib>
#include <mutex>

#include "bcf_kernels.cuh"
#include "bcf_merge_tma.cuh"
#include "bcf_merge_win.cuh"
#include "bcf_launch.h"

namespace bcf {

// Opt in to > 48 KB dynamic shared memory once per (kernel, device).  The
// once-flag must be distinct per kernel instantiation: it lives in the
// caller's template (not in a helper templated only on the function type).
template <typename K>
cudaError_t ensure_smem_attr(K kernel, size_t bytes, int& done_mask) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (bytes <= 48 * 1024 || (__atomic_load_n(&done_mask, __ATOMIC_ACQUIRE) >> dev) & 1) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) __atomic_fetch_or(&done_mask, 1 << dev, __ATOMIC_ACQ_REL);
  else (void)cudaGetLastError();  // do not leave a stale error for the next launch check
  return e;
}

// Launch with programmatic dependent launch (PDL): consecutive passes of a
// sort overlap their launch latency and CTA ramp-up with the previous pass's
// tail; every kernel waits (griddepcontrol.wait) before touching global
// memory.  BCF_NO_PDL=1 launches plainly (A/B measurements).
inline bool pdl_enabled() {
  static const bool on = [] {
    const char* v = getenv("BCF_NO_PDL");
    return !(v && v[0] == '1');
  }();
  return on;
}

template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kern)(KArgs...), unsigned grid, unsigned block, size_t smem, cudaStream_t s,
                     Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, args...);
}

template <int E, int U, bool PAIRS, bool CF>
cudaError_t launch_block_sort(const SortArgs& a, long long grid, cudaStream_t s) {
  constexpr size_t smem = tile_smem_bytes<E, U, PAIRS>();
  static int done = 0, done_loop = 0;
  if (a.ntiles > 0) {  // grid-stride measurement mode
    cudaError_t e = ensure_smem_attr(block_sort_kernel<E, U, PAIRS, CF, true>, smem, done_loop);
    if (e != cudaSuccess) return e;
    return launch_k(block_sort_kernel<E, U, PAIRS, CF, true>, (unsigned)grid, U, smem, s, a);
  }
  cudaError_t e = ensure_smem_attr(block_sort_kernel<E, U, PAIRS, CF>, smem, done);
  if (e != cudaSuccess) return e;
  return launch_k(block_sort_kernel<E, U, PAIRS, CF>, (unsigned)grid, U, smem, s, a);
}

template <int E, int U>
cudaError_t launch_block_sort2(const SortArgs& a, long long grid, cudaStream_t s) {
  constexpr size_t smem = (size_t)tile2_words<E, U>() * sizeof(uint32_t);
  static int done = 0;
  cudaError_t e = ensure_smem_attr(block_sort2_kernel<E, U>, smem, done);
  if (e != cudaSuccess) return e;
  return launch_k(block_sort2_kernel<E, U>, (unsigned)grid, U, smem, s, a);
}

template <int E, int U, bool PAIRS, bool CF, bool BDESC>
cudaError_t launch_merge(const MergeArgs& a, long long grid, cudaStream_t s) {
  constexpr size_t smem = tile_smem_bytes<E, U, PAIRS>();
  static int done = 0, done_loop = 0;
  if (a.ntiles > 0) {  // grid-stride measurement mode
    cudaError_t e = ensure_smem_attr(merge_pass_kernel<E, U, PAIRS, CF, BDESC, true>, smem, done_loop);
    if (e != cudaSuccess) return e;
    return launch_k(merge_pass_kernel<E, U, PAIRS, CF, BDESC, true>, (unsigned)grid, U, smem, s, a);
  }
  cudaError_t e = ensure_smem_attr(merge_pass_kernel<E, U, PAIRS, CF, BDESC>, smem, done);
  if (e != cudaSuccess) return e;
  return launch_k(merge_pass_kernel<E, U, PAIRS, CF, BDESC>, (unsigned)grid, U, smem, s, a);
}

// persistent TMA merge pass: grid = min(tiles, SMs x resident CTAs), each
// CTA a contiguous, balanced chunk of tiles
struct PersistentCache {
  // filled once per device under `mu`; per_sm is published last (release)
  // and read first (acquire), so a reader that sees it non-zero sees nsm
  int per_sm[32] = {0};
  int nsm[32] = {0};
  std::mutex mu;
};

template <typename K>
cudaError_t launch_persistent(K kern, PersistentCache& pc, size_t smem, int threads, const MergeArgs& a,
                              long long tiles, cudaStream_t s) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev >= 32) return cudaErrorInvalidDevice;
  if (__atomic_load_n(&pc.per_sm[dev], __ATOMIC_ACQUIRE) == 0) {
    std::lock_guard<std::mutex> lk(pc.mu);
    if (pc.per_sm[dev] == 0) {
      if (smem > 48 * 1024) {
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) {
          (void)cudaGetLastError();
          return e;
        }
      }
      int k = 0, sms = 0;
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&k, kern, threads, smem);
      if (e != cudaSuccess) return e;
      e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
      if (e != cudaSuccess) return e;
      pc.nsm[dev] = sms;
      __atomic_store_n(&pc.per_sm[dev], k > 0 ? k : 1, __ATOMIC_RELEASE);
    }
  }
  // one wave of SMs x resident CTAs, tiles spread evenly (per_cta = 0)
  long long ctas = (long long)pc.nsm[dev] * pc.per_sm[dev];
  if (ctas > tiles) ctas = tiles;
  return launch_k(kern, (unsigned)ctas, (unsigned)threads, smem, s, a, tiles, 0ll);
}

#ifndef BCF_MERGE_WIN
#define BCF_MERGE_WIN 1
#endif
// BCF_PAIRS_TMA=1: pairs passes on the 3-stage exact-split TMA kernel instead
// of the window kernel (A/B measurements)
inline bool pairs_tma_forced() {
  static const bool on = [] {
    const char* v = getenv("BCF_PAIRS_TMA");
    return v && v[0] == '1';
  }();
  return on;
}

template <int E, int U, bool PAIRS>
cudaError_t launch_merge_tma(const MergeArgs& a, long long tiles, cudaStream_t s) {
  static PersistentCache pc;  // one per (E, U, PAIRS) instantiation
  // the 2-stage window ring (x2 for pairs) must fit in 227 KB; otherwise the
  // 3-stage exact-split TMA kernel
  constexpr bool win_fits = win_smem_bytes<E, U, PAIRS>() <= 227 * 1024;
  if constexpr (BCF_MERGE_WIN && win_fits) {
    if (!PAIRS || !pairs_tma_forced())
      return launch_persistent(merge_pass_win_kernel<E, U, PAIRS>, pc, win_smem_bytes<E, U, PAIRS>(), U + 32, a,
                               tiles, s);
  }
  static PersistentCache pc_tma;
  return launch_persistent(merge_pass_tma_kernel<E, U, PAIRS>, pc_tma, tma_smem_bytes<E, U, PAIRS>(), U + 32, a,
                           tiles, s);
}

// the window kernel alone (keys only; bcf_merge_u32 passes B through src_kb,
// which only the window and plain kernels read)
template <int E, int U, bool PAIRS>
cudaError_t launch_merge_win(const MergeArgs& a, long long tiles, cudaStream_t s) {
  static PersistentCache pc;
  return launch_persistent(merge_pass_win_kernel<E, U, PAIRS>, pc, win_smem_bytes<E, U, PAIRS>(), U + 32, a, tiles,
                           s);
}

// every regular pass of a sort in one launch (MergeArgs::npass, progress flags)
template <int E, int U, bool PAIRS>
cudaError_t launch_merge_multi(const MergeArgs& a, long long tiles, cudaStream_t s) {
  static PersistentCache pc;
  return launch_persistent(merge_pass_win_kernel<E, U, PAIRS, true>, pc, win_smem_bytes<E, U, PAIRS>(), U + 32, a, tiles,
                           s);
}

inline bool even_window_enabled() {
  const char* v = getenv("BCF_EVEN_WIN");
  return v && v[0] == '1';
}

template <int E, int U>
void register_eu(LaunchTable& t) {
  const int ui = u_index(U);
  t.v[E][ui][0][0] = {&launch_block_sort<E, U, false, true>, &launch_merge<E, U, false, true, true>,
                      &launch_merge<E, U, false, true, false>};
  t.v[E][ui][0][1] = {&launch_block_sort<E, U, true, true>, &launch_merge<E, U, true, true, true>,
                      &launch_merge<E, U, true, true, false>};
  t.v[E][ui][1][0] = {&launch_block_sort<E, U, false, false>, &launch_merge<E, U, false, false, false>,
                      nullptr};
  if constexpr (cgcd(W, E) > 1) {
    // rho != identity: the window kernel with cp.async staging in rho's
    // physical order and LSU copy-out is opt-in (BCF_EVEN_WIN=1): the one-CTA-
    // per-tile kernel with physical-order LSU staging by every thread is faster
    // for every even E (2^27: 530-800 vs 800-2240 us per pass,
    // profiles/r02_evenE_plain_vs_window_2p27.txt).  (The general (MULTI)
    // instantiation: faster here than the one-pass one, 795 vs 875 us.)
    if (even_window_enabled()) {
      if constexpr (BCF_MERGE_WIN && win_smem_bytes<E, U>() <= 227 * 1024)
        t.v[E][ui][0][0].merge_tma = &launch_merge_multi<E, U, false>;
      if constexpr (BCF_MERGE_WIN && win_smem_bytes<E, U, true>() <= 227 * 1024)
        t.v[E][ui][0][1].merge_tma = &launch_merge_multi<E, U, true>;
    }
  }
  if constexpr (cgcd(W, E) == 1 && E + 1 == W && U == 256) t.v[E][ui][0][0].block_sort2 = &launch_block_sort2<E, U>;
  if constexpr (cgcd(W, E) == 1) {
    t.v[E][ui][0][0].merge_tma = &launch_merge_tma<E, U, false>;
    t.v[E][ui][0][1].merge_tma = &launch_merge_tma<E, U, true>;
    if constexpr (BCF_MERGE_WIN && win_smem_bytes<E, U>() <= 227 * 1024) {
      t.v[E][ui][0][0].merge_win = &launch_merge_win<E, U, false>;
      t.v[E][ui][0][0].merge_multi = &launch_merge_multi<E, U, false>;
    }
    if constexpr (BCF_MERGE_WIN && win_smem_bytes<E, U, true>() <= 227 * 1024) {
      t.v[E][ui][0][1].merge_win = &launch_merge_win<E, U, true>;
      t.v[E][ui][0][1].merge_multi = &launch_merge_multi<E, U, true>;
    }
  }
}

}  // namespace bcf

// BCF_ONLY_E / BCF_ONLY_U (A/B experiment builds): instantiate one (E, u)
#ifndef BCF_ONLY_U
#define BCF_REG_U(E, U) register_eu<E, U>(t);
#else
#define BCF_REG_U(E, U) \
  if constexpr (U == BCF_ONLY_U) register_eu<E, U>(t);
#endif
#define BCF_DEFINE_REG(E)                         \
  namespace bcf {                                 \
  void register_E##E(LaunchTable& t) {            \
    if constexpr (BCF_E_ENABLED(E)) {             \
      BCF_REG_U(E, 128)                           \
      BCF_REG_U(E, 256)                           \
      BCF_REG_U(E, 512)                           \
    }                                             \
  }                                               \
  }
#ifdef BCF_ONLY_E
#define BCF_E_ENABLED(E) ((E) == BCF_ONLY_E)
#else
#define BCF_E_ENABLED(E) true
#endif
