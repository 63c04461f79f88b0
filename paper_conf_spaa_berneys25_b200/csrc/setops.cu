// setops.cu -- set operations of two ascending u32 sequences (multiset
// semantics of ISO C++ [alg.set.operations]) on top of the CF merge: the
// paper's generalisation "any algorithm that involves a parallel scan of a
// pair of arrays".  bcf_set_op_u32 (bcf_capi.cu) runs
//   1. tags: A element i -> i, B element j -> 0x80000000 | j;
//   2. the stable CF merge of (A, tags) and (B, tags) (bcf_merge_u32, ties to
//      A, conflict-free staging and gather);
//   3. keep flags over the merged sequence M: in the run of equal keys x
//      (m copies from A first, then n from B, by stability), the A copy of
//      rank k and the B copy of rank k are kept by
//        union          A always,  B iff k >= m  (the last n - m of B's)
//        intersection   A iff k < n
//        difference     A iff k >= n            (the last m - n of A's)
//        symmetric      A iff k >= n, B iff k >= m;
//      run bounds by exponential + binary search around each position (one
//      or two loads for short runs), the A/B boundary of a run by binary
//      search on the tags;
//   4. compaction: per-block keep counts, one-block exclusive scan, scatter
//      of the kept keys (and their tags) in merged order.
#include <cuda_runtime.h>

#include <cstdint>

namespace bcf {
namespace setops {

constexpr int THREADS = 256;
constexpr int ITEMS = 16;
constexpr long long BLK = (long long)THREADS * ITEMS;

__global__ void tags_kernel(uint32_t* __restrict__ ta, long long na, uint32_t* __restrict__ tb, long long nb) {
  const long long n = na + nb;
  for (long long q = blockIdx.x * (long long)blockDim.x + threadIdx.x; q < n; q += (long long)gridDim.x * blockDim.x) {
    if (q < na) ta[q] = (uint32_t)q;
    else tb[q - na] = 0x80000000u | (uint32_t)(q - na);
  }
}

// first index in [lo, p] with M[i] == x (M ascending, M[p] == x)
__device__ __forceinline__ long long run_begin(const uint32_t* __restrict__ M, long long p, uint32_t x) {
  long long step = 1, hi = p;  // M[hi] == x
  long long lo = p;
  while (true) {
    const long long c = p - step;
    if (c < 0) { lo = -1; break; }
    if (__ldg(M + c) != x) { lo = c; break; }  // M[lo] != x
    hi = c;
    step <<= 1;
  }
  // answer in (lo, hi]: first index with M == x
  while (hi - lo > 1) {
    const long long mid = lo + ((hi - lo) >> 1);
    if (__ldg(M + mid) == x) hi = mid; else lo = mid;
  }
  return hi;
}

// one past the last index with M[i] == x (M[p] == x)
__device__ __forceinline__ long long run_end(const uint32_t* __restrict__ M, long long n, long long p, uint32_t x) {
  long long step = 1, lo = p;  // M[lo] == x
  long long hi = p;
  while (true) {
    const long long c = p + step;
    if (c >= n) { hi = n; break; }
    if (__ldg(M + c) != x) { hi = c; break; }
    lo = c;
    step <<= 1;
  }
  while (hi - lo > 1) {
    const long long mid = lo + ((hi - lo) >> 1);
    if (__ldg(M + mid) == x) lo = mid; else hi = mid;
  }
  return hi;
}

// first index in [b, e) whose tag marks a B element (tags A...A B...B in a run)
__device__ __forceinline__ long long first_b(const uint32_t* __restrict__ V, long long b, long long e) {
  long long lo = b, hi = e;
  while (lo < hi) {
    const long long mid = lo + ((hi - lo) >> 1);
    if (__ldg(V + mid) & 0x80000000u) hi = mid; else lo = mid + 1;
  }
  return lo;
}

__device__ __forceinline__ bool keep(int op, const uint32_t* __restrict__ M, const uint32_t* __restrict__ V,
                                     long long n, long long p) {
  const uint32_t x = __ldg(M + p);
  const bool isB = (__ldg(V + p) & 0x80000000u) != 0;
  // fast path: a run of one (no equal neighbour)
  const bool left = p > 0 && __ldg(M + p - 1) == x;
  const bool right = p + 1 < n && __ldg(M + p + 1) == x;
  long long p0, p1, pb;
  if (!left && !right) {
    p0 = p;
    p1 = p + 1;
    pb = isB ? p : p + 1;
  } else {
    p0 = left ? run_begin(M, p, x) : p;
    p1 = right ? run_end(M, n, p, x) : p + 1;
    pb = first_b(V, p0, p1);
  }
  const long long m = pb - p0, nB = p1 - pb;  // copies in A, in B
  if (!isB) {
    const long long k = p - p0;
    switch (op) {
      case 0: return true;
      case 1: return k < nB;
      default: return k >= nB;  // difference, symmetric difference
    }
  }
  const long long k = p - pb;
  return (op == 0 || op == 3) && k >= m;
}

// keep bits of a block's BLK merged positions, striped: bit q of thread t is
// position base + q * THREADS + t (every load of a row is coalesced)
__device__ __forceinline__ uint32_t keep_bits(int op, const uint32_t* __restrict__ M, const uint32_t* __restrict__ V,
                                              long long n, long long base) {
  uint32_t mask = 0;
#pragma unroll 4
  for (int q = 0; q < ITEMS; ++q) {
    const long long p = base + (long long)q * THREADS + threadIdx.x;
    if (p < n && keep(op, M, V, n, p)) mask |= 1u << q;
  }
  return mask;
}

// per-block keep counts
__global__ void __launch_bounds__(THREADS) count_kernel(int op, const uint32_t* __restrict__ M,
                                                        const uint32_t* __restrict__ V, long long n,
                                                        unsigned long long* __restrict__ counts) {
  int c = __popc(keep_bits(op, M, V, n, blockIdx.x * BLK));
  for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
  __shared__ int ws[THREADS / 32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int t = 0;
    for (int w = 0; w < THREADS / 32; ++w) t += ws[w];
    counts[blockIdx.x] = (unsigned long long)t;
  }
}

// exclusive scan of nb block counts in place (one CTA); total -> *total
__global__ void __launch_bounds__(1024) scan_kernel(unsigned long long* __restrict__ counts, long long nb,
                                                    unsigned long long* __restrict__ total) {
  const int t = threadIdx.x;
  const long long per = (nb + 1023) / 1024;
  const long long b0 = t * per, b1 = b0 + per < nb ? b0 + per : nb;
  unsigned long long s = 0;
  for (long long b = b0; b < b1; ++b) s += counts[b];
  __shared__ unsigned long long sh[1024];
  sh[t] = s;
  __syncthreads();
  for (int o = 1; o < 1024; o <<= 1) {  // inclusive Hillis-Steele scan
    const unsigned long long v = t >= o ? sh[t - o] : 0ull;
    __syncthreads();
    sh[t] += v;
    __syncthreads();
  }
  unsigned long long run = t ? sh[t - 1] : 0ull;
  for (long long b = b0; b < b1; ++b) {
    const unsigned long long c = counts[b];
    counts[b] = run;
    run += c;
  }
  if (t == 1023) *total = sh[1023];
}

__global__ void __launch_bounds__(THREADS) scatter_kernel(int op, const uint32_t* __restrict__ M,
                                                          const uint32_t* __restrict__ V, long long n,
                                                          const unsigned long long* __restrict__ offsets,
                                                          uint32_t* __restrict__ out, uint32_t* __restrict__ out_src) {
  constexpr int NWARP = THREADS / 32;
  const long long base = blockIdx.x * BLK;
  const uint32_t mask = keep_bits(op, M, V, n, base);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // kept count of every (row q, warp w) segment, then their exclusive scan in
  // merged order (row-major: position base + q THREADS + 32 w + lane)
  __shared__ int seg[ITEMS * NWARP];
  uint32_t bal[ITEMS];
#pragma unroll
  for (int q = 0; q < ITEMS; ++q) {
    bal[q] = __ballot_sync(0xffffffffu, (mask >> q) & 1u);
    if (lane == 0) seg[q * NWARP + warp] = __popc(bal[q]);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int k = 0; k < ITEMS * NWARP; ++k) {
      const int c = seg[k];
      seg[k] = run;
      run += c;
    }
  }
  __syncthreads();
  const unsigned long long o0 = offsets[blockIdx.x];
  const uint32_t lt = (1u << lane) - 1u;
#pragma unroll
  for (int q = 0; q < ITEMS; ++q) {
    if ((mask >> q) & 1u) {
      const long long p = base + (long long)q * THREADS + threadIdx.x;
      const unsigned long long o = o0 + (unsigned long long)(seg[q * NWARP + warp] + __popc(bal[q] & lt));
      out[o] = __ldg(M + p);
      if (out_src) out_src[o] = __ldg(V + p);
    }
  }
}

// launches 3 and 4 (the flags, scan and scatter kernels); M, V merged keys
// and tags of n elements; counts: nblocks + 1 words of temp
cudaError_t compact(int op, const uint32_t* M, const uint32_t* V, long long n, unsigned long long* counts,
                    unsigned long long* d_count, uint32_t* out, uint32_t* out_src, cudaStream_t s) {
  const long long nb = (n + BLK - 1) / BLK;
  if (nb == 0) return cudaMemsetAsync(d_count, 0, sizeof(unsigned long long), s);
  count_kernel<<<(unsigned)nb, THREADS, 0, s>>>(op, M, V, n, counts);
  scan_kernel<<<1, 1024, 0, s>>>(counts, nb, d_count);
  scatter_kernel<<<(unsigned)nb, THREADS, 0, s>>>(op, M, V, n, counts, out, out_src);
  return cudaGetLastError();
}

long long compact_blocks(long long n) { return (n + BLK - 1) / BLK; }

cudaError_t make_tags(uint32_t* ta, long long na, uint32_t* tb, long long nb, cudaStream_t s) {
  const long long n = na + nb;
  if (n == 0) return cudaSuccess;
  const long long blocks = (n + 255) / 256 < 148LL * 16 ? (n + 255) / 256 : 148LL * 16;
  tags_kernel<<<(unsigned)blocks, 256, 0, s>>>(ta, na, tb, nb);
  return cudaGetLastError();
}

}  // namespace setops
}  // namespace bcf
