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
//   4. compaction in one pass (decoupled look-back over per-block keep
//      counts), scatter of the kept keys (and their tags) in merged order.
#include <cuda_runtime.h>

#include <cstdint>

namespace bcf {
namespace setops {

#ifndef BCF_LB_SLEEP_NS
#define BCF_LB_SLEEP_NS 100
#endif
#ifndef BCF_SETOP_THREADS
#define BCF_SETOP_THREADS 256
#endif
constexpr int THREADS = BCF_SETOP_THREADS;
#ifndef BCF_SETOP_ITEMS
#define BCF_SETOP_ITEMS 16
#endif
constexpr int ITEMS = BCF_SETOP_ITEMS;
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


// the keep rule for a copy at merged position p of the run [p0, p1) whose B
// copies start at pb (m = pb - p0 copies from A, nB = p1 - pb from B)
__device__ __forceinline__ bool keep_rule(int op, bool isB, long long p, long long p0, long long pb, long long p1) {
  const long long m = pb - p0, nB = p1 - pb;
  if (!isB) {
    const long long k = p - p0;
    return op == 0 ? true : (op == 1 ? k < nB : k >= nB);
  }
  return (op == 0 || op == 3) && p - pb >= m;
}

// keep bits of a block's BLK merged positions, striped: bit q of thread t is
// position base + q * THREADS + t (every load of a row is coalesced).  A warp
// row covers 32 consecutive positions: the run bounds and the A/B boundary of
// a run that starts and ends inside the row come from three ballots (run
// heads, run tails, B copies); only runs crossing the row's edge search
// global memory (run_begin / run_end / first_b).
__device__ __forceinline__ uint32_t keep_bits(int op, const uint32_t* __restrict__ M, const uint32_t* __restrict__ V,
                                              long long n, long long base) {
  const int lane = threadIdx.x & 31;
  const bool full = base + BLK <= n;      // every position of the block exists (all but the last block)
  const bool after_ok = base + BLK < n;   // the position after the block exists
  const uint32_t* __restrict__ Mb = M + base;
  const uint32_t* __restrict__ Vb = V + base;
  uint32_t mask = 0;
#pragma unroll 4
  for (int q = 0; q < ITEMS; ++q) {
    const int o = q * THREADS + (int)threadIdx.x;  // offset in the block
    const bool in = full || base + o < n;
    const uint32_t x = in ? __ldg(Mb + o) : 0u;
    const bool isB = in && (__ldg(Vb + o) & 0x80000000u) != 0;
    uint32_t xp = __shfl_up_sync(0xffffffffu, x, 1);
    uint32_t xn = __shfl_down_sync(0xffffffffu, x, 1);
    if (lane == 0) xp = (in && (o > 0 || base > 0)) ? __ldg(Mb + o - 1) : ~x;
    const bool next_ok = full ? (o + 1 < BLK || after_ok) : (base + o + 1 < n);
    if (lane == 31 || !next_ok) xn = (in && next_ok) ? __ldg(Mb + o + 1) : ~x;
    const bool head = in && xp != x;  // (xp = ~x before position 0)
    const bool tail = in && xn != x;  // (xn = ~x after position n-1)
    const unsigned H = __ballot_sync(0xffffffffu, head);
    const unsigned Tl = __ballot_sync(0xffffffffu, tail);
    const unsigned Bm = __ballot_sync(0xffffffffu, isB);
    if (!in) continue;
    const unsigned upto = lane == 31 ? 0xffffffffu : ((2u << lane) - 1u);  // lanes 0..lane
    const unsigned hs = H & upto, te = Tl & ~((1u << lane) - 1u);
    bool k;
    if (hs && te) {
      // the run is lanes [l0, l1] of this row; its B copies start at lane lb
      const int l0 = 31 - __clz(hs), l1 = __ffs(te) - 1;
      const unsigned inrun = (l1 == 31 ? 0xffffffffu : ((2u << l1) - 1u)) & ~((1u << l0) - 1u);
      const unsigned bb = Bm & inrun;
      const int lb = bb ? __ffs(bb) - 1 : l1 + 1;
      if (isB) {
        k = (op == 0 || op == 3) && lane - lb >= lb - l0;
      } else {
        const int kk = lane - l0, nB = l1 + 1 - lb;
        k = op == 0 ? true : (op == 1 ? kk < nB : kk >= nB);
      }
    } else {
      // the run crosses the row's edge: bounds from global memory
      const long long p = base + o, row0 = p - lane;
      const long long p0 = hs ? row0 + (31 - __clz(hs)) : run_begin(M, p, x);
      const long long p1 = te ? row0 + __ffs(te) : run_end(M, n, p, x);
      const long long pb = first_b(V, p0, p1);
      k = keep_rule(op, isB, p, p0, pb, p1);
    }
    if (k) mask |= 1u << q;
  }
  return mask;
}

// single-pass compaction (decoupled look-back): blocks take tiles in order
// from a counter, publish their keep count (AGGREGATE) at once, then walk
// back over their predecessors' words until an inclusive PREFIX, publish
// their own PREFIX and scatter.  status[b] = flag << 62 | value (0 = not
// ready); the last tile writes the total.
constexpr unsigned long long ST_AGG = 1ull << 62, ST_PRE = 2ull << 62, ST_VAL = (1ull << 62) - 1;

__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

#ifndef BCF_SETOP_MINB
#define BCF_SETOP_MINB 8  // 8 blocks per SM (32 registers): the look-back waits are latency, more blocks hide them (858 -> 745 us at 2 x 2^25)
#endif
__global__ void __launch_bounds__(THREADS, BCF_SETOP_MINB) compact_lookback_kernel(int op, const uint32_t* __restrict__ M,
                                                                   const uint32_t* __restrict__ V, long long n,
                                                                   unsigned long long* __restrict__ status,
                                                                   unsigned int* __restrict__ ticket,
                                                                   unsigned long long* __restrict__ total,
                                                                   uint32_t* __restrict__ out,
                                                                   uint32_t* __restrict__ out_src) {
  constexpr int NWARP = THREADS / 32;
  __shared__ long long s_tile;
  __shared__ int seg[ITEMS * NWARP];
  __shared__ unsigned long long s_excl;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const long long b = s_tile;
  const long long nb = (n + BLK - 1) / BLK;
  const long long base = b * BLK;
  const uint32_t mask = keep_bits(op, M, V, n, base);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t bal[ITEMS];
#pragma unroll
  for (int q = 0; q < ITEMS; ++q) {
    bal[q] = __ballot_sync(0xffffffffu, (mask >> q) & 1u);
    if (lane == 0) seg[q * NWARP + warp] = __popc(bal[q]);
  }
  __syncthreads();
  if (warp == 0) {
    // exclusive scan of the ITEMS * NWARP segment counts (4 per lane)
    int v[ITEMS * NWARP / 32];
    int sum = 0;
#pragma unroll
    for (int k = 0; k < ITEMS * NWARP / 32; ++k) {
      v[k] = seg[lane * (ITEMS * NWARP / 32) + k];
      sum += v[k];
    }
    int inc = sum;
    for (int o = 1; o < 32; o <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += t;
    }
    int run = inc - sum;
#pragma unroll
    for (int k = 0; k < ITEMS * NWARP / 32; ++k) {
      seg[lane * (ITEMS * NWARP / 32) + k] = run;
      run += v[k];
    }
    const unsigned long long cnt = (unsigned long long)__shfl_sync(0xffffffffu, inc, 31);
    // publish, then look back
    unsigned long long excl = 0;
    if (b == 0) {
      if (lane == 0) st_rel(status, ST_PRE | cnt);
    } else {
      if (lane == 0) st_rel(status + b, ST_AGG | cnt);
      long long k0 = b - 1;  // window [k0 - 31, k0]
      while (true) {
        const long long k = k0 - lane;
        unsigned long long w = k >= 0 ? ld_acq(status + k) : ST_PRE;  // before tile 0: prefix 0
        const unsigned ready = __ballot_sync(0xffffffffu, w != 0ull);
        const unsigned pre = __ballot_sync(0xffffffffu, (w & ~ST_VAL) == ST_PRE);
        const int first_pre = pre ? __ffs(pre) - 1 : 32;  // nearest prefix in the window
        const unsigned need = first_pre < 31 ? ((2u << first_pre) - 1u) : 0xffffffffu;
        if ((ready & need) != need) {  // a predecessor not yet published: back off, re-read
          __nanosleep(BCF_LB_SLEEP_NS);
          continue;
        }
        unsigned long long add = (lane <= first_pre && k >= 0) ? (w & ST_VAL) : 0ull;
        for (int o = 16; o > 0; o >>= 1) add += __shfl_xor_sync(0xffffffffu, add, o);
        excl += add;
        if (first_pre < 32) break;
        k0 -= 32;
      }
      if (lane == 0) st_rel(status + b, ST_PRE | (excl + cnt));
    }
    if (lane == 0) {
      s_excl = excl;
      if (b == nb - 1) *total = excl + cnt;
    }
  }
  __syncthreads();
  const unsigned long long o0 = s_excl;
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
// counts: nblocks + 1 words of temp (look-back status words + the ticket)
cudaError_t compact(int op, const uint32_t* M, const uint32_t* V, long long n, unsigned long long* counts,
                    unsigned long long* d_count, uint32_t* out, uint32_t* out_src, cudaStream_t s) {
  const long long nb = (n + BLK - 1) / BLK;
  if (nb == 0) return cudaMemsetAsync(d_count, 0, sizeof(unsigned long long), s);
  cudaError_t e = cudaMemsetAsync(counts, 0, (size_t)(nb + 1) * sizeof(unsigned long long), s);
  if (e != cudaSuccess) return e;
  compact_lookback_kernel<<<(unsigned)nb, THREADS, 0, s>>>(op, M, V, n, counts, (unsigned int*)(counts + nb),
                                                           d_count, out, out_src);
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
