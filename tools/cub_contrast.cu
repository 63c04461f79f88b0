// cub_contrast.cu -- SURVEY §8(f) row f4: the paper's Fig. 5/6 contrast on B200
// with a real library.  Times CUB's DeviceMergeSort (the Thrust/CUB pairwise
// mergesort the paper analyses; on sm_100 CUB's
// MaxPolicy is Policy600 = 256 threads x 17 items for 4-byte keys) on
// uniform-random keys and on the worst-case input our generator builds for
// ITS (E, u) = (17, 256) (Section 4), next to bcf_sort_u32
// (CF, defaults) on the same two inputs in the same process.  Context, not a
// target: no oracle is used; outputs are cross-checked (CUB == bcf, sorted).
//
// Timing: CUDA events on one stream, L2 flushed (256 MiB memset) before every
// rep outside the events, random / worst-case interleaved (ABAB), median.
//
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a
//        tools/cub_contrast.cu -Iinclude -Lpaper_conf_spaa_berneys25_b200 -lbcf
//        -Xlinker -rpath -Xlinker $PWD/paper_conf_spaa_berneys25_b200 -o tools/cub_contrast
// Run:   tools/cub_contrast [log2n=24 | n] [reps=20]   -> one JSON line on stdout
#include <cub/device/device_merge_sort.cuh>
#include <cub/device/device_radix_sort.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "bcf.h"

#define CK(x)                                                                       \
  do {                                                                              \
    cudaError_t e_ = (x);                                                           \
    if (e_ != cudaSuccess) {                                                        \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      exit(1);                                                                      \
    }                                                                               \
  } while (0)
#define BK(x)                                                                       \
  do {                                                                              \
    bcf_status s_ = (x);                                                            \
    if (s_ != BCF_SUCCESS) {                                                        \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, bcf_status_string(s_)); \
      exit(1);                                                                      \
    }                                                                               \
  } while (0)

struct Less {
  __host__ __device__ bool operator()(uint32_t a, uint32_t b) const { return a < b; }
};

// synthetic_inputs.py recipe: h_i = mix64(seed + (i+1) * golden), key = hi32
static uint64_t mix64(uint64_t z) {
  z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27; z *= 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static double median(std::vector<double> v) {
  std::sort(v.begin(), v.end());
  return v[v.size() / 2];
}

int main(int argc, char** argv) {
  const long long arg = argc > 1 ? atoll(argv[1]) : 24;  // log2(n) if <= 40, else n
  const int reps = argc > 2 ? atoi(argv[2]) : 20;
  const uint64_t n = arg <= 40 ? 1ull << arg : (uint64_t)arg;
  const uint64_t seed = 0xB2000000ull + 1;  // BASELINE configs[1]
  std::vector<uint32_t> h_rand(n), h_worst(n), h_a(n), h_b(n);
  for (uint64_t i = 0; i < n; ++i) h_rand[i] = (uint32_t)(mix64(seed + (i + 1) * 0x9E3779B97F4A7C15ull) >> 32);
  BK(bcf_worst_case_u32_host(h_worst.data(), n, 17, 256, seed));  // CUB's own (E, u)

  uint32_t *d_rand, *d_worst, *d_out, *d_flush;
  const size_t flush_bytes = 256ull << 20;
  CK(cudaMalloc(&d_rand, n * 4));
  CK(cudaMalloc(&d_worst, n * 4));
  CK(cudaMalloc(&d_out, n * 4));
  CK(cudaMalloc(&d_flush, flush_bytes));
  CK(cudaMemcpy(d_rand, h_rand.data(), n * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_worst, h_worst.data(), n * 4, cudaMemcpyHostToDevice));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));

  size_t cub_merge_bytes = 0, cub_radix_bytes = 0, bcf_bytes = 0;
  CK(cub::DeviceMergeSort::SortKeysCopy(nullptr, cub_merge_bytes, d_rand, d_out, (int64_t)n, Less{}, s));
  CK(cub::DeviceRadixSort::SortKeys(nullptr, cub_radix_bytes, d_rand, d_out, (int64_t)n, 0, 32, s));
  BK(bcf_sort_u32(d_rand, d_out, n, nullptr, &bcf_bytes, nullptr, s));
  const size_t tb = std::max({cub_merge_bytes, cub_radix_bytes, bcf_bytes});
  void* d_temp;
  CK(cudaMalloc(&d_temp, tb));

  enum { CUB_MERGE, CUB_RADIX, BCF_CF, NIMPL };
  const char* names[NIMPL] = {"cub_merge_sort", "cub_radix_sort", "bcf_sort_u32"};
  auto run = [&](int impl, const uint32_t* in) {
    size_t t = tb;
    if (impl == CUB_MERGE) CK(cub::DeviceMergeSort::SortKeysCopy(d_temp, t, in, d_out, (int64_t)n, Less{}, s));
    else if (impl == CUB_RADIX) CK(cub::DeviceRadixSort::SortKeys(d_temp, t, in, d_out, (int64_t)n, 0, 32, s));
    else BK(bcf_sort_u32(in, d_out, n, d_temp, &t, nullptr, s));
  };

  // correctness: all three agree on both inputs and are sorted
  for (int which = 0; which < 2; ++which) {
    const uint32_t* in = which ? d_worst : d_rand;
    run(BCF_CF, in);
    CK(cudaMemcpyAsync(h_a.data(), d_out, n * 4, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    for (uint64_t i = 1; i < n; ++i)
      if (h_a[i - 1] > h_a[i]) { fprintf(stderr, "bcf output not sorted at %llu\n", (unsigned long long)i); return 1; }
    for (int impl : {CUB_MERGE, CUB_RADIX}) {
      run(impl, in);
      CK(cudaMemcpyAsync(h_b.data(), d_out, n * 4, cudaMemcpyDeviceToHost, s));
      CK(cudaStreamSynchronize(s));
      if (h_a != h_b) { fprintf(stderr, "%s disagrees with bcf\n", names[impl]); return 1; }
    }
  }

  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  std::vector<double> ms[NIMPL][2];
  for (int rep = -3; rep < reps; ++rep)
    for (int which = 0; which < 2; ++which)  // ABAB
      for (int impl = 0; impl < NIMPL; ++impl) {
        CK(cudaMemsetAsync(d_flush, rep & 0xFF, flush_bytes, s));
        CK(cudaEventRecord(e0, s));
        run(impl, which ? d_worst : d_rand);
        CK(cudaEventRecord(e1, s));
        CK(cudaEventSynchronize(e1));
        float t;
        CK(cudaEventElapsedTime(&t, e0, e1));
        if (rep >= 0) ms[impl][which].push_back(t);
      }

  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, 0));
  printf("{\"tool\": \"cub_contrast\", \"n\": %llu, \"reps\": %d, \"gpu\": \"%s\", \"cuda_runtime_cub\": %d, "
         "\"worst_case\": \"bcf_worst_case_u32_host(n, E=17, u=256) = CUB Policy600 (256 threads x 17 items)\", "
         "\"l2\": \"flushed (256 MiB memset) before every rep, outside the events\", \"results\": {",
         (unsigned long long)n, reps, prop.name, CUB_VERSION);
  for (int impl = 0; impl < NIMPL; ++impl) {
    const double r = median(ms[impl][0]), w = median(ms[impl][1]);
    printf("%s\"%s\": {\"random_ms\": %.5f, \"worst_ms\": %.5f, \"random_keys_per_s\": %.6g, "
           "\"worst_keys_per_s\": %.6g, \"worst_over_random_time\": %.4f}",
           impl ? ", " : "", names[impl], r, w, n / (r * 1e-3), n / (w * 1e-3), w / r);
  }
  printf("}}\n");
  return 0;
}
