// bcf_kernels.cuh -- the three hot-path kernels of the pairwise mergesort
// (PAPER.md:59-61, :348-354), each in two variants:
//   CF       the paper's bank-conflict-free design (pi + rho layout, Alg. 1
//            gather, conflict-free split search, in-register merge network);
//   BASELINE the unmodified Thrust design the paper measures against
//            (A|B forward in shared memory, per-thread binary merge path,
//            serial merge reading shared memory) -- keys only.
//
// block_sort  one CTA sorts a tile of T = U*E keys: per-thread sort of E keys,
//             then log2(U) merge levels in shared memory.
// merge_pass  one CTA produces one output tile of T keys of a pairwise merge
//             of runs of R keys (merge-path tile split fused in).
//
// Global run directions (CF only): in every pass run r is stored descending
// iff r is odd, so a tile's B range, read with unit stride, lands in shared
// memory already reversed (pi).  The final run (index 0) is
// ascending.  The baseline keeps every run ascending.
#pragma once
#include "bcf_device.cuh"
#include "bcf_tma.cuh"

namespace bcf {

constexpr uint32_t PAD_KEY = 0xffffffffu;

// dynamic shared memory of one CTA
// T keys + E words of slack (cell-scan probes past the end, see
// lane_split_smem) + 1 (the serial merge's look-ahead load in the baseline)
template <int E, int U>
__host__ __device__ constexpr int tile_words() {
  return U * E + E + 1;
}
template <int E, int U, bool PAIRS>
__host__ __device__ constexpr size_t tile_smem_bytes() {
  return (size_t)tile_words<E, U>() * sizeof(uint32_t) * (PAIRS ? 2 : 1);
}

struct SortArgs {
  const uint32_t* in_k;
  const uint32_t* in_v;
  uint32_t* out_k;
  uint32_t* out_v;
  long long n;
  int encode_f32;  // encode f32 -> totalOrder u32 on load (block sort)
  int decode_f32;  // decode on the final store
  int cf_dirs;     // CF run directions (odd runs descending)
  unsigned int* zero;  // if set, block 0 zeroes zero[0, nzero) (the next launch's progress flags)
  int nzero;
  long long ntiles;    // > 0: a grid smaller than the tile count loops over tiles (grid stride)
};

// One merge group: A = src[a_off, a_off+na), B = src[b_off, b_off+nb),
// output dst[out_off, out_off+na+nb); *_desc: run stored descending.
struct GroupDesc {
  long long a_off, na, b_off, nb, out_off, tile_begin;
  int a_desc, b_desc, out_desc, pad_;
  // plain kernel, keys only: A / B keys read from these bases (any device or
  // peer-mapped pointer, bcf_merge_runs_ptrs_u32) instead of src_k / src_kb
  const uint32_t* a_ptr;
  const uint32_t* b_ptr;
};

struct MergeArgs {
  const uint32_t* src_k;
  const uint32_t* src_v;
  uint32_t* dst_k;
  uint32_t* dst_v;
  long long n;
  long long R;     // input run length (regular mode)
  int log2_tpg;    // log2(2R / T): tiles per group (regular mode)
  int decode_f32;  // final pass of an f32 sort
  int cf_dirs;     // regular mode: odd runs descending
  const GroupDesc* groups;  // table mode (merge of arbitrary runs) if non-null
  int ngroups;
  unsigned long long* trace;  // debug timeline (BCF_TRACE), nullptr normally
  // table mode (plain and window kernels): B runs read from these bases
  // instead of src_k / src_v (bcf_merge_u32: A and B in separate arrays;
  // bcf_merge_runs_u32 pass 1: B runs reversed into temp); nullptr = same
  const uint32_t* src_kb;
  const uint32_t* src_vb;
  // multi-pass mode (persistent window kernel, regular passes only): npass
  // consecutive passes in one launch.  Pass p reads buf_k[p & 1] (src_k is
  // ignored), writes buf_k[(p + 1) & 1] or, for the last pass, dst_k; run
  // length R << p, log2_tpg + p; decode_f32 applies to the last pass.  Pass p
  // of a CTA starts once every CTA whose tiles cover its input groups has
  // published progress[cta] >= p (zeroed before the launch).
  int npass;
  unsigned int* progress;
  uint32_t* buf_k[2];
  uint32_t* buf_v[2];
  long long ntiles;  // plain kernel: > 0 -> grid-stride loop over this many tiles
};

// Group of output tile `tile`: regular pairwise pass (run 2g with run 2g+1,
// run r descending iff r odd under CF directions) or an explicit table.
__device__ __forceinline__ GroupDesc group_of_tile(const MergeArgs& args, long long tile, int T,
                                                   long long& j) {
  GroupDesc G;
  if (args.groups == nullptr) {
    const long long g = tile >> args.log2_tpg;  // tiles per group = 2R/T = 2^log2_tpg
    j = tile - (g << args.log2_tpg);
    const long long g0 = g * 2 * args.R;
    const long long left = args.n - g0;
    G.a_off = g0;
    G.na = left < args.R ? left : args.R;
    G.nb = left - G.na < args.R ? left - G.na : args.R;
    // descending runs of length L < R are stored shifted by sigma = (R-L) mod 4
    // so that a tile's A range and B range share one 16-byte phase (TMA path)
    G.b_off = g0 + args.R + (args.cf_dirs ? ((args.R - G.nb) & 3) : 0);
    G.tile_begin = g << args.log2_tpg;
    G.a_desc = 0;
    G.b_desc = args.cf_dirs;
    G.out_desc = args.cf_dirs && (g & 1);
    G.out_off = g0 + (G.out_desc ? ((2 * args.R - G.na - G.nb) & 3) : 0);
    G.pad_ = 0;
    G.a_ptr = nullptr;
    G.b_ptr = nullptr;
  } else {
    int lo = 0, hi = args.ngroups - 1;  // last group with tile_begin <= tile
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (args.groups[mid].tile_begin <= tile) lo = mid; else hi = mid - 1;
    }
    G = args.groups[lo];
    j = tile - G.tile_begin;
  }
  return G;
}

// ---------------------------------------------------------------------------
// Output stage shared by both kernels: registers -> shared (round sets, rho
// layout) -> coalesced global stores.  Thread's items are tile outputs
// [D, D+E); `desc` writes the tile mirrored into a descending run whose
// global element o lives at c0 + (T-1-o) ... expressed as gaddr = c0 + q with
// q the logical smem index.
// ---------------------------------------------------------------------------
template <int E, int U, bool PAIRS>
__device__ __forceinline__ void store_tile(uint32_t* sk, uint32_t* sv, const uint32_t (&key)[E],
                                           const uint32_t (&val)[E], int D, int cnt, bool desc,
                                           uint32_t* __restrict__ gk, uint32_t* __restrict__ gv,
                                           long long c0, bool decode) {
  constexpr int T = U * E;
  // round m: ascending -> item m at D+m; descending -> item E-1-m at T-E-D+m
  if (desc) {
#pragma unroll
    for (int m = 0; m < E; ++m) {
      const int idx = rho<E>(T - E - D + m);
      sk[idx] = key[E - 1 - m];
      if constexpr (PAIRS) sv[idx] = val[E - 1 - m];
    }
  } else {
#pragma unroll
    for (int m = 0; m < E; ++m) {
      const int idx = rho<E>(D + m);
      sk[idx] = key[m];
      if constexpr (PAIRS) sv[idx] = val[m];
    }
  }
  const int qlo = desc ? T - cnt : 0;
  const int qhi = desc ? T : cnt;
  uint32_t* __restrict__ pk = gk + c0;
  uint32_t* __restrict__ pv = PAIRS ? gv + c0 : nullptr;
  // (LSU stores, not a bulk copy: a bulk shared->global copy running beside
  // other CTAs' shared-memory instructions shows up in the unit-level bank
  // conflict counter -- 0.68 M per 2^24 block sort)
  __syncthreads();
  if constexpr (cgcd(W, E) == 1 && !PAIRS && (T % 4) == 0) {
    // a full tile into a 16-byte aligned run (rho = identity: physical order is
    // the output order): 16-byte loads and stores, a quarter-warp reads 128
    // consecutive bytes (one wavefront, no conflict)
    if (cnt == T && !decode && (((uintptr_t)pk) & 15) == 0) {
      for (int q = 4 * (int)threadIdx.x; q < T; q += 4 * U)
        *reinterpret_cast<uint4*>(pk + q) = *reinterpret_cast<const uint4*>(sk + q);
      return;
    }
  }
  if (decode) {
#pragma unroll
    for (int r = 0; r < E; ++r) {
      const int P = threadIdx.x + r * U;  // physical word: consecutive per warp
      const int q = rho_inv<E>(P);
      if (q >= qlo && q < qhi) {
        pk[q] = f32_decode(sk[P]);
        if constexpr (PAIRS) pv[q] = sv[P];
      }
    }
  } else {
#pragma unroll
    for (int r = 0; r < E; ++r) {
      const int P = threadIdx.x + r * U;
      const int q = rho_inv<E>(P);
      if (q >= qlo && q < qhi) {
        pk[q] = sk[P];
        if constexpr (PAIRS) pv[q] = sv[P];
      }
    }
  }
}

// ---------------------------------------------------------------------------
// Block sort (K1): tile t of T = U*E input keys -> sorted run t (descending
// iff t odd under CF directions).
// ---------------------------------------------------------------------------
#ifndef BCF_BS_MINB256
#define BCF_BS_MINB256 0  // 0: no min-blocks hint (ptxas picks ~80 registers, 3 CTAs/SM)
#endif
#ifndef BCF_BS_MINB512
#define BCF_BS_MINB512 0
#endif
#ifndef BCF_BS_PAIRS_MINB256
#define BCF_BS_PAIRS_MINB256 5  // pairs (11, 256): <= 51 registers, 5 CTAs/SM (ptxas alone picks 64)
#endif
template <int U, bool PAIRS = false, int E = 0>
__host__ __device__ constexpr int bs_min_blocks() {
  // (the pairs cap spills at E >= 15: those keep ptxas's choice)
  return (PAIRS && U == 256 && E <= 13) ? BCF_BS_PAIRS_MINB256
                                        : (U == 256 ? BCF_BS_MINB256 : (U == 512 ? BCF_BS_MINB512 : 0));
}

// The block sort of one tile of T = U*E keys (input t0 .. t0+cnt of
// args.in_k, pads = max key): on return, thread tid holds the sorted tile's
// outputs [tid E, tid E + E) in key[] (val[] for pairs); sk / sv (tile_words
// each) are its working buffers, still being read by other threads until the
// caller's next __syncthreads.
#ifndef BCF_WARP_PAD
#define BCF_WARP_PAD 1
#endif
#ifndef BCF_WARP_POW2
#define BCF_WARP_POW2 1
#endif
template <int E, int U, bool PAIRS, bool CF>
__device__ __forceinline__ void block_sort_core(const SortArgs& args, uint32_t* sk, uint32_t* sv,
                                                const long long t0, const int cnt, uint32_t (&key)[E],
                                                uint32_t (&val)[E]) {
  constexpr int NW = U / W;
  __shared__ int s_org[NW + 1];
  const int tid = threadIdx.x;
  const int lane = tid & (W - 1);
  const int warp = tid >> 5;

  // keys only, E = 31: levels 0..4 (runs up to one warp) run in registers
  // across the warp (warp_bitonic_levels); any assignment of the warp's 992
  // keys to its lanes works, so each lane loads its keys straight from global
  // memory (coalesced: key r of lane l is element 32 r + l of the warp's
  // chunk) without the shared-memory round trip of the general path
  // (also E = 16 and 8: E slots per lane, no pad, the warp runs written
  // through rho; BCF_WARP_POW2=0 keeps those on the shared-memory levels)
  // (and E < 16 other than 8: 16 slots per lane with max-key pads; BCF_WARP_PAD=0: off)
  constexpr bool WARP_PAD = CF && !PAIRS && BCF_WARP_PAD && E < 16 && E != 8;
  constexpr bool WARP_PHASE =
      CF && !PAIRS && U >= 2 * W && (E + 1 == W || (BCF_WARP_POW2 && (E == 16 || E == 8)) || WARP_PAD);
  uint32_t tag[E];
  if constexpr (WARP_PHASE) {
    const int wbase = warp * (W * E);
    const uint32_t* __restrict__ gin_k = args.in_k + t0 + wbase + lane;
    const int lim = cnt - wbase - lane;  // element 32 r + lane exists iff 32 r < lim
    if (lim >= W * E) {  // a full warp chunk (every tile but the last): no predicates
#pragma unroll
      for (int r = 0; r < E; ++r) key[r] = __ldg(gin_k + W * r);
    } else {
#pragma unroll
      for (int r = 0; r < E; ++r) key[r] = (W * r < lim) ? __ldg(gin_k + W * r) : PAD_KEY;
    }
    if (args.encode_f32) {
#pragma unroll
      for (int r = 0; r < E; ++r)
        if (W * r < lim) key[r] = f32_encode(key[r]);
    }
  } else {
    // --- load: coalesced in physical order, pads = max key (they sort last and
    // are trimmed by the count; stable order keeps them after real max keys).
    {
      const uint32_t* __restrict__ gin_k = args.in_k + t0;
      const uint32_t* __restrict__ gin_v = PAIRS ? args.in_v + t0 : nullptr;
      uint32_t vk[E], vv[E];
#pragma unroll
      for (int r = 0; r < E; ++r) {
        const int P = tid + r * U;
        const int p = CF ? rho_inv<E>(P) : P;
        vk[r] = PAD_KEY;
        vv[r] = 0;
        if (p < cnt) {
          vk[r] = __ldg(gin_k + p);
          if constexpr (PAIRS) vv[r] = __ldg(gin_v + p);
        }
      }
      if (args.encode_f32) {
#pragma unroll
        for (int r = 0; r < E; ++r) {
          const int P = tid + r * U;
          const int p = CF ? rho_inv<E>(P) : P;
          if (p < cnt) vk[r] = f32_encode(vk[r]);
        }
      }
#pragma unroll
      for (int r = 0; r < E; ++r) {
        sk[tid + r * U] = vk[r];
        if constexpr (PAIRS) sv[tid + r * U] = vv[r];
      }
    }
    __syncthreads();
    // blocked read: round m reads logical tid*E + m (a round set)
#pragma unroll
    for (int m = 0; m < E; ++m) {
      const int idx = CF ? rho<E>(tid * E + m) : tid * E + m;
      key[m] = sk[idx];
      if constexpr (PAIRS) { val[m] = sv[idx]; tag[m] = m; }
    }
  }
  oddeven_sort_pad<E, PAIRS>(key, tag, val);

  // warp phase, then the warp runs go to shared memory in the level-5 layout
  // and the CF shared-memory levels continue from l = 5
  int l_first = 0;
  if constexpr (WARP_PHASE && E + 1 == W) {
    uint32_t k32[W];
#pragma unroll
    for (int i = 0; i < E; ++i) k32[i] = key[i];
    k32[E] = PAD_KEY;
#ifndef BCF_TIMING_SKIP_WARP
    warp_bitonic_levels<W>(k32, lane);
#endif
    __syncthreads();  // (general path: every thread has finished its blocked read of sk)
    warp_run_scatter<E>(sk, k32, warp, lane);
    l_first = 5;
  } else if constexpr (WARP_PHASE && WARP_PAD) {
    uint32_t k16[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) k16[i] = i < E ? key[i] : PAD_KEY;
    warp_bitonic_levels<16>(k16, lane);
    __syncthreads();
    warp_run_scatter_rho_pad<E>(sk, k16, warp, lane);
    l_first = 5;
  } else if constexpr (WARP_PHASE) {
    warp_bitonic_levels<E>(key, lane);
    __syncthreads();
    warp_run_scatter_rho<E>(sk, key, warp, lane);
    l_first = 5;
  }
#ifdef BCF_TIMING_SKIP_LEVELS
  l_first = 30;  // timing-only build: no shared-memory levels (wrong output)
#endif

  // --- log2(U) merge levels: runs of S = E*2^l, groups of G = 2^(l+1) threads
#pragma unroll 1
  for (int l = l_first; (1 << l) < U; ++l) {
    const int S = E << l;
    const int G = 2 << l;
    const int ir = tid & ((1 << l) - 1);   // index within its run
    const int run = tid >> l;
    const int gbase = (run >> 1) * 2 * S;  // group base (logical)
    const bool isB = run & 1;
    __syncthreads();
    if (WARP_PHASE && l == 5) {
      // the warp runs were written by warp_run_scatter
    } else if constexpr (CF) {
      // conflict-free scatter (fn. 5): B runs are written
      // reversed (pi); in round m B-run lanes write item E-1-m so that every
      // lane writes logical index = m (mod E).  From l = 5 on a run spans
      // whole warps, so the A/B choice is warp-uniform.
      const int base = isB ? gbase + 2 * S - E - ir * E : gbase + ir * E;
      if ((1 << l) >= W) {
        if (isB) {
#pragma unroll
          for (int m = 0; m < E; ++m) {
            const int idx = rho<E>(base + m);
            sk[idx] = key[E - 1 - m];
            if constexpr (PAIRS) sv[idx] = val[E - 1 - m];
          }
        } else {
#pragma unroll
          for (int m = 0; m < E; ++m) {
            const int idx = rho<E>(base + m);
            sk[idx] = key[m];
            if constexpr (PAIRS) sv[idx] = val[m];
          }
        }
      } else {
#pragma unroll
        for (int m = 0; m < E; ++m) {
          const int idx = rho<E>(base + m);
          sk[idx] = isB ? key[E - 1 - m] : key[m];
          if constexpr (PAIRS) sv[idx] = isB ? val[E - 1 - m] : val[m];
        }
      }
    } else {
      const int base = gbase + (isB ? S : 0) + ir * E;
#pragma unroll
      for (int m = 0; m < E; ++m) sk[base + m] = key[m];
    }
    __syncthreads();
    const int ig = tid & (G - 1);
    const int D = ig * E;
    if constexpr (CF) {
      int alpha = 0, Dw = 0, WL = G, nit = l + 1;
      if (G > W) {
        Dw = (ig >> 5) * (W * E);
        alpha = warp_origin_smem<E>(sk, gbase, 2 * S, S, S, Dw, lane);
        WL = W;
        nit = 5;
        if (lane == 0) s_org[warp] = alpha;
        __syncthreads();  // uniform: G depends on l only
      }
      const int a = lane_split_smem<E>(sk, gbase, 2 * S, S, S, Dw, alpha, lane, WL, nit);
      int anext = __shfl_down_sync(FULL, a, 1);
      if ((lane & (WL - 1)) == WL - 1) {
        // last lane of the window: next window's origin, or the group end
        anext = (G > W && ((ig >> 5) + 1) * W < G) ? s_org[warp + 1] : S;
      }
      const int nA = anext - a;
      const int nB = E - nA;
      const int b = D - a;
      dual_subsequence_gather<E, PAIRS, true>(sk, sv, gbase, 2 * S, a, b, nA, nB, key, val, PAD_KEY);
      merge_registers<E, PAIRS>(key, val, a, nA, nB);
    } else {
      // unmodified Thrust: per-thread binary merge path, then serial merge
      // reading shared memory
      const int abase = gbase, bbase = gbase + S;
      int lo = D - S < 0 ? 0 : D - S;
      int hi = D < S ? D : S;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (sk[bbase + D - 1 - mid] < sk[abase + mid]) hi = mid; else lo = mid + 1;
      }
      int ab = abase + lo, bb = bbase + (D - lo);
      const int ae = abase + S, be = bbase + S;
      uint32_t k1 = sk[ab], k2 = sk[bb];
#pragma unroll
      for (int m = 0; m < E; ++m) {
        const bool p = (bb < be) && ((ab >= ae) || (k2 < k1));
        key[m] = p ? k2 : k1;
        if (p) ++bb; else ++ab;
        const uint32_t x = sk[p ? bb : ab];
        if (p) k2 = x; else k1 = x;
      }
    }
  }
}

template <int E, int U, bool PAIRS, bool CF>
__device__ __forceinline__ void block_sort_tile(const SortArgs& args, const long long tile) {
  constexpr int T = U * E;
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  uint32_t* sk = smem_dyn;                      // tile_words keys
  uint32_t* sv = smem_dyn + tile_words<E, U>(); // tile_words values (pairs only)
  const int tid = threadIdx.x;
  const long long t0 = tile * T;
  const long long rem = args.n - t0;
  const int cnt = rem < T ? (int)rem : T;
  tma::pdl_wait();  // the input may be produced by the preceding grid
  // (after the wait: the preceding grid may be a merge launch using the flags)
  if (args.zero != nullptr && tile == 0)
    for (int k = tid; k < args.nzero; k += U) args.zero[k] = 0u;
  uint32_t key[E], val[E];
  block_sort_core<E, U, PAIRS, CF>(args, sk, sv, t0, cnt, key, val);
  __syncthreads();
  tma::pdl_trigger();  // the next pass may be scheduled once this wave ends
  // --- store run `tile`: descending iff tile odd (CF directions)
  const bool desc = args.cf_dirs && (tile & 1);
  // a short descending run is stored shifted by sigma = (T - cnt) mod 4
  const long long c0 = desc ? t0 + ((T - cnt) & 3) + cnt - T : t0;
  store_tile<E, U, PAIRS>(sk, sv, key, val, tid * E, cnt, desc, args.out_k, args.out_v, c0,
                          args.decode_f32 != 0);
}

// ---------------------------------------------------------------------------
// Two-tile block sort (keys only, CF, E coprime with w; SURVEY.md §8(f) f3,
// fewer HBM passes): one CTA sorts the tiles 2p and 2p+1 (T = U*E keys each)
// with block_sort_core, keeps them in shared memory as one merge group of the
// paper's layout (tile 2p ascending at [0, T), tile 2p+1 reversed (pi) at
// [T, 2T)), and merges them with one more conflict-free level in two rounds
// of T outputs (warp origins, lane splits, Alg. 1 gather, register merge):
// runs of 2T leave the kernel, so the sort needs one merge pass fewer.
// ---------------------------------------------------------------------------
template <int E, int U>
__host__ __device__ constexpr int tile2_words() {
  return 2 * U * E + E + 1;
}

template <int E, int U>
__device__ __forceinline__ void block_sort2_tile(const SortArgs& args, const long long pair) {
  static_assert(cgcd(W, E) == 1, "two-tile block sort: rho = identity");
  constexpr int T = U * E;
  constexpr int T2 = 2 * T;
  constexpr int NW = U / W;
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  uint32_t* sk = smem_dyn;  // tile2_words keys
  __shared__ int s_org2[2][NW + 1];
  const int tid = threadIdx.x;
  const int lane = tid & (W - 1);
  const int warp = tid >> 5;
  const long long t0 = pair * T2;
  const long long rem = args.n - t0;
  const int cntA = rem < T ? (int)rem : T;
  const int cntB = rem - T <= 0 ? 0 : (rem - T < T ? (int)(rem - T) : T);
  tma::pdl_wait();
  if (args.zero != nullptr && pair == 0)
    for (int k = tid; k < args.nzero; k += U) args.zero[k] = 0u;
  uint32_t key[E], val[E];
  const bool desc = args.cf_dirs && (pair & 1);
  const int ntile = cntB > 0 ? 2 : 1;
  // one copy of the block-sort code for both tiles (instruction cache)
#pragma unroll 1
  for (int h = 0; h < ntile; ++h) {
    block_sort_core<E, U, false, true>(args, sk + h * T, sk + h * T, t0 + h * T, h ? cntB : cntA, key, val);
    __syncthreads();  // every thread has finished reading the tile's buffer
    if (ntile == 1) break;
    // tile 2p -> A at [0, T) ascending (round m writes tid E + m, a round
    // set); tile 2p+1 -> B reversed, B[y] at 2T-1-y (a short B stays anchored
    // at the group end, reading c17; round m writes 2T-1-tid E-m)
    const int base = h ? T2 - 1 - tid * E : tid * E;
    const int step = h ? -1 : 1;
#pragma unroll
    for (int m = 0; m < E; ++m) sk[base + step * m] = key[m];
  }
  if (ntile == 1) {
    // the last, short run: one tile
    tma::pdl_trigger();
    const long long c0 = desc ? t0 + ((T - cntA) & 3) + cntA - T : t0;
    store_tile<E, U, false>(sk, sk, key, val, tid * E, cntA, desc, args.out_k, args.out_v, c0,
                            args.decode_f32 != 0);
    return;
  }
  __syncthreads();
  // one more CF merge level over the group (NA = T, NB = cntB), two rounds
  const int NA = T, NB = cntB, cnt2 = T + cntB;
  uint32_t key0[E];
#pragma unroll 1
  for (int r = 0; r < 2; ++r) {
    const int Dw = r * T + warp * W * E;
    const int alpha = warp_origin_smem<E>(sk, 0, T2, NA, NB, Dw, lane);
    if (lane == 0) s_org2[r][warp] = alpha;
    if (warp == 0) {
      const int aend = r == 0 ? warp_origin_smem<E>(sk, 0, T2, NA, NB, T, lane) : NA;
      if (lane == 0) s_org2[r][NW] = aend;
    }
    __syncthreads();
    const int D = r * T + tid * E;
    int a = lane_split_smem<E>(sk, 0, T2, NA, NB, Dw, alpha, lane, W, 5);
    if (D >= cnt2) a = NA;
    int anext = __shfl_down_sync(FULL, a, 1);
    if (lane == W - 1) anext = (Dw + W * E >= cnt2) ? NA : s_org2[r][warp + 1];
    const int Dc = D < cnt2 ? D : cnt2;
    const int Dn = D + E < cnt2 ? D + E : cnt2;
    const int nA = anext - a;
    const int nB = (Dn - Dc) - nA;
    const int b = Dc - a;
    if (cnt2 == T2)
      dual_subsequence_gather<E, false, true>(sk, sk, 0, T2, a, b, nA, nB, key, val, PAD_KEY);
    else
      dual_subsequence_gather<E, false, false>(sk, sk, 0, T2, a, b, nA, nB, key, val, PAD_KEY);
    merge_registers<E, false>(key, val, a, nA, nB);
    if (r == 0) {
#pragma unroll
      for (int m = 0; m < E; ++m) key0[m] = key[m];
    }
  }
  __syncthreads();
  tma::pdl_trigger();
  // --- store the run of 2T (descending iff the pair index is odd; a short
  // descending run shifted by sigma = (2T - cnt2) mod 4): round-set STS of
  // both rounds' outputs, then coalesced stores
  const int D0 = tid * E, D1 = T + tid * E;
  if (desc) {
#pragma unroll
    for (int m = 0; m < E; ++m) sk[T2 - E - D0 + m] = key0[E - 1 - m];
#pragma unroll
    for (int m = 0; m < E; ++m) sk[T2 - E - D1 + m] = key[E - 1 - m];
  } else {
#pragma unroll
    for (int m = 0; m < E; ++m) sk[D0 + m] = key0[m];
#pragma unroll
    for (int m = 0; m < E; ++m) sk[D1 + m] = key[m];
  }
  __syncthreads();
  const long long c0 = desc ? t0 + ((T2 - cnt2) & 3) + cnt2 - T2 : t0;
  const int qlo = desc ? T2 - cnt2 : 0;
  const int qhi = desc ? T2 : cnt2;
  uint32_t* __restrict__ pk = args.out_k + c0;
  if (args.decode_f32) {
    for (int q = qlo + tid; q < qhi; q += U) pk[q] = f32_decode(sk[q]);
    return;
  }
  // consecutive words per warp: conflict-free loads, coalesced stores
#pragma unroll 4
  for (int q = qlo + tid; q < qhi; q += U) pk[q] = sk[q];
}

template <int E, int U>
__global__ void __launch_bounds__(U, bs_min_blocks<U>()) block_sort2_kernel(SortArgs args) {
  block_sort2_tile<E, U>(args, blockIdx.x);
}

// ---------------------------------------------------------------------------
// Merge pass (K2+K3 fused): output tile `blockIdx.x` of the pairwise merge of
// runs of R keys.  Group g merges run 2g (A) with run 2g+1 (B).
// ---------------------------------------------------------------------------
// LOOP: a grid smaller than the tile count loops over the tiles (grid stride,
// the one-CTA-per-SM measurement mode, SortArgs::ntiles).  A separate
// instantiation: the loop raises ptxas's register choice for the whole kernel
// (block_sort<31, 256> 80 -> 128 registers, 138 -> 146 us at 2^24).
template <int E, int U, bool PAIRS, bool CF, bool LOOP = false>
__global__ void __launch_bounds__(U, bs_min_blocks<U, PAIRS, E>()) block_sort_kernel(SortArgs args) {
  if constexpr (!LOOP) {
    block_sort_tile<E, U, PAIRS, CF>(args, blockIdx.x);
  } else {
    const long long nt = args.ntiles > 0 ? args.ntiles : (long long)gridDim.x;
    for (long long t = blockIdx.x; t < nt; t += gridDim.x) {
      if (t != blockIdx.x) __syncthreads();  // the previous tile's copy-out has read shared memory
      block_sort_tile<E, U, PAIRS, CF>(args, t);
    }
  }
}

template <int E, int U, bool PAIRS, bool CF, bool BDESC>
__device__ __forceinline__ void merge_pass_tile(const MergeArgs& args, const long long tile) {
  constexpr int T = U * E;
  constexpr int NW = U / W;
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  uint32_t* sk = smem_dyn;                      // tile_words keys
  uint32_t* sv = smem_dyn + tile_words<E, U>(); // tile_words values (pairs only)
  __shared__ int s_org[NW + 1];
  __shared__ long long s_split[2];
  const int tid = threadIdx.x;
  const int lane = tid & (W - 1);
  const int warp = tid >> 5;
  tma::pdl_wait();  // pass i reads what pass i-1 wrote (and overwrites what it read)
  long long j;
  const GroupDesc grp = group_of_tile(args, tile, T, j);
  const long long lenG = grp.na + grp.nb;
  const uint32_t* __restrict__ baseAk = grp.a_ptr ? grp.a_ptr : args.src_k;
  const uint32_t* __restrict__ baseBk = grp.b_ptr ? grp.b_ptr : (args.src_kb ? args.src_kb : args.src_k);
  RunView Av{baseAk + grp.a_off, grp.na, grp.a_desc};
  RunView Bv{baseBk + grp.b_off, grp.nb, grp.b_desc};
  const long long D0 = j * T;
  const long long D1 = D0 + T < lenG ? D0 + T : lenG;

  // --- tile split by warp-cooperative merge path over global memory
  if (warp < 2) {
    const long long D = warp == 0 ? D0 : D1;
    const long long a = merge_path_warp_global(Av, Bv, D, lane);
    if (lane == 0) s_split[warp] = a;
  }
  __syncthreads();
  const long long a0 = s_split[0];
  const long long a1 = s_split[1];
  const int cnt = (int)(D1 - D0);
  const int NA = (int)(a1 - a0);
  const int NB = cnt - NA;
  const long long b0 = D0 - a0;

  // --- staging: A forward at logical [0, NA); B reversed (CF: B[y] at T-1-y)
  // or forward behind A (baseline).  Physical-order, coalesced global reads;
  // element q of A at oA + sA*q, element y of B at oB' +- y (pointer math once).
  {
    // A runs are ascending: A element (a0 + q) at a_off + a0 + q.
    // CF: logical q >= T-NB holds B[y], y = b0 + T-1-q; B stored descending
    //     (BDESC, regular passes) at b_off + nb-1-y = (b_off + nb-b0-T) + q,
    //     or ascending (table mode) at b_off + y = (b_off + b0+T-1) - q.
    // baseline: logical q in [NA, cnt) holds B[b0 + q - NA] (ascending).
    constexpr int sB = (CF && !BDESC) ? -1 : 1;
    const long long oA = grp.a_off + a0;
    const long long oB = CF ? (BDESC ? grp.b_off + grp.nb - b0 - T : grp.b_off + b0 + T - 1)
                            : grp.b_off + b0 - NA;
    const uint32_t* __restrict__ pAk = baseAk + oA;
    const uint32_t* __restrict__ pBk = baseBk + oB;
    const uint32_t* __restrict__ pAv = PAIRS ? args.src_v + oA : nullptr;
    const uint32_t* __restrict__ pBv = PAIRS ? (args.src_vb ? args.src_vb : args.src_v) + oB : nullptr;
    const int bstart = CF ? T - NB : NA;
    const int bend = CF ? T : cnt;
    uint32_t vk[E], vv[E];
#pragma unroll
    for (int r = 0; r < E; ++r) {
      const int P = tid + r * U;
      const int q = CF ? rho_inv<E>(P) : P;
      const bool isA = q < NA;
      const bool isB = q >= bstart && q < bend;
      vk[r] = 0;
      vv[r] = 0;
      if (isA) {
        vk[r] = __ldg(pAk + q);
        if constexpr (PAIRS) vv[r] = __ldg(pAv + q);
      }
      if (isB) {
        vk[r] = __ldg(pBk + sB * q);
        if constexpr (PAIRS) vv[r] = __ldg(pBv + sB * q);
      }
    }
#pragma unroll
    for (int r = 0; r < E; ++r) {
      const int P = tid + r * U;
      const int q = CF ? rho_inv<E>(P) : P;
      if (q < NA || (q >= bstart && q < bend)) {
        sk[P] = vk[r];
        if constexpr (PAIRS) sv[P] = vv[r];
      }
    }
  }
  __syncthreads();

  uint32_t key[E], val[E];
  const int D = tid * E;
  if constexpr (CF) {
    const int Dw = warp * W * E;
    const int alpha = warp_origin_smem<E>(sk, 0, T, NA, NB, Dw, lane);
    if (lane == 0) s_org[warp] = alpha;
    if (tid == 0) s_org[NW] = NA;
    __syncthreads();
    const int a = lane_split_smem<E>(sk, 0, T, NA, NB, Dw, alpha, lane, W, 5);
    int anext = __shfl_down_sync(FULL, a, 1);
    if (lane == W - 1) anext = s_org[warp + 1];
    const int Dc = D < cnt ? D : cnt;
    const int Dn = D + E < cnt ? D + E : cnt;
    const int nA = anext - a;
    const int nB = (Dn - Dc) - nA;
    const int b = Dc - a;
    if (cnt == T)
      dual_subsequence_gather<E, PAIRS, true>(sk, sv, 0, T, a, b, nA, nB, key, val, PAD_KEY);
    else
      dual_subsequence_gather<E, PAIRS, false>(sk, sv, 0, T, a, b, nA, nB, key, val, PAD_KEY);
    merge_registers<E, PAIRS>(key, val, a, nA, nB);
  } else {
    if (D < cnt) {
      int lo = D - NB < 0 ? 0 : D - NB;
      int hi = D < NA ? D : NA;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (sk[NA + D - 1 - mid] < sk[mid]) hi = mid; else lo = mid + 1;
      }
      int ab = lo, bb = NA + (D - lo);
      const int ae = NA, be = NA + NB;
      uint32_t k1 = sk[ab], k2 = sk[bb];
#pragma unroll
      for (int m = 0; m < E; ++m) {
        const bool p = (bb < be) && ((ab >= ae) || (k2 < k1));
        key[m] = p ? k2 : k1;
        if (p) ++bb; else ++ab;
        const uint32_t x = sk[p ? bb : ab];
        if (p) k2 = x; else k1 = x;
      }
    } else {
#pragma unroll
      for (int m = 0; m < E; ++m) key[m] = PAD_KEY;
    }
  }
  __syncthreads();
  tma::pdl_trigger();
  // --- output tile into the group's output run (descending if grp.out_desc)
  const bool desc = grp.out_desc != 0;
  const long long c0 = desc ? grp.out_off + lenG - D0 - T : grp.out_off + D0;
  store_tile<E, U, PAIRS>(sk, sv, key, val, D, cnt, desc, args.dst_k, args.dst_v, c0,
                          args.decode_f32 != 0);
}

// LOOP: as for block_sort_kernel (MergeArgs::ntiles, grid-stride over tiles)
template <int E, int U, bool PAIRS, bool CF, bool BDESC, bool LOOP = false>
__global__ void __launch_bounds__(U) merge_pass_kernel(MergeArgs args) {
  if constexpr (!LOOP) {
    merge_pass_tile<E, U, PAIRS, CF, BDESC>(args, blockIdx.x);
  } else {
    const long long nt = args.ntiles > 0 ? args.ntiles : (long long)gridDim.x;
    for (long long t = blockIdx.x; t < nt; t += gridDim.x) {
      if (t != blockIdx.x) __syncthreads();
      merge_pass_tile<E, U, PAIRS, CF, BDESC>(args, t);
    }
  }
}

}  // namespace bcf
