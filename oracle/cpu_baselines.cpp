// oracle/cpu_baselines.cpp -- TEST INFRASTRUCTURE / CPU BASELINES ONLY.
//
// The two further CPU baselines SURVEY.md §8(d) asks for beside the plain
// oracle (sort_oracle.c), timed by bench.py's cpu_baseline leg on the GPU
// box's host cores, and used by tests/ as an independent cross-check of the
// oracle (library routine):
//   (ii)  std::stable_sort of n u32 keys on ONE core;
//   (iii) a parallel stable mergesort on `threads` cores: the input is split
//         into `threads` contiguous chunks, each sorted by std::stable_sort in
//         its own std::thread, then a merge tree of std::merge (left run first
//         on ties, so the result is the stable order) with the independent
//         merges of one level in parallel.
// Shares no code with the CUDA path; never linked by the product.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

extern "C" {

int baseline_std_stable_sort_u32(const uint32_t* in, uint32_t* out, uint64_t n) {
  std::memcpy(out, in, n * sizeof(uint32_t));
  std::stable_sort(out, out + n);
  return 0;
}

int baseline_parallel_mergesort_u32(const uint32_t* in, uint32_t* out, uint64_t n, int threads) {
  if (threads < 1) threads = 1;
  if (n < (uint64_t)threads * 1024) threads = 1;
  std::vector<uint32_t> tmp(n);
  std::memcpy(out, in, n * sizeof(uint32_t));
  std::vector<uint64_t> cut(threads + 1);
  for (int t = 0; t <= threads; ++t) cut[t] = n * (uint64_t)t / threads;
  {
    std::vector<std::thread> th;
    for (int t = 0; t < threads; ++t)
      th.emplace_back([&, t] { std::stable_sort(out + cut[t], out + cut[t + 1]); });
    for (auto& x : th) x.join();
  }
  // merge tree: runs [cut[i], cut[i+1]) pairwise, level by level
  std::vector<uint64_t> runs(cut);
  uint32_t* src = out;
  uint32_t* dst = tmp.data();
  while (runs.size() > 2) {
    std::vector<uint64_t> next;
    std::vector<std::thread> th;
    for (size_t i = 0; i + 1 < runs.size(); i += 2) {
      const uint64_t a = runs[i], b = runs[i + 1];
      const uint64_t c = (i + 2 < runs.size()) ? runs[i + 2] : b;
      next.push_back(a);
      th.emplace_back([=] {
        if (c > b) std::merge(src + a, src + b, src + b, src + c, dst + a);
        else std::memcpy(dst + a, src + a, (b - a) * sizeof(uint32_t));
      });
    }
    next.push_back(n);
    for (auto& x : th) x.join();
    std::swap(src, dst);
    runs.swap(next);
  }
  if (src != out) std::memcpy(out, src, n * sizeof(uint32_t));
  return 0;
}

}  // extern "C"
