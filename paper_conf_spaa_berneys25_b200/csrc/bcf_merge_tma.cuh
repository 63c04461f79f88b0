// bcf_merge_tma.cuh -- persistent, warp-specialised CF merge pass for
// coprime E (d = 1, rho = identity).
//
// One CTA = U consumer threads (NW warps) + 1 producer warp, looping over a
// contiguous chunk of output tiles with a TMA_STAGES-deep shared-memory ring:
//   producer  merge-path split of the next tile (warp-cooperative 32-ary
//             search over global memory; consecutive tiles reuse the previous
//             boundary, so only ~3 rounds over a range <= T), then two 1-D
//             bulk copies (TMA engine) bring the tile's A range and B range
//             (B runs are stored descending, so the range lands reversed = pi)
//             into the stage at a common word shift c = 16-byte phase of the
//             source; at most 6 misaligned edge words are copied by lanes.
//             Completion is tracked by an mbarrier (expect_tx).  When the
//             consumers have written a tile's outputs back into its stage,
//             the producer streams them out with a bulk store.
//   consumers the conflict-free in-tile merge of bcf_device.cuh (warp
//             origin, lane split, Alg. 1 gather, register merge), then the
//             output round-set stores into the stage (shifted by the output's
//             16-byte phase) and an mbarrier arrive.
// The layout seen by the consumers is exactly the paper's rho(A u pi(B))
// with rho = id, offset by the constant c (a constant shift preserves every
// round set's bank pattern).
//
// Alignment: A runs start at multiples of 4 words and B runs
// are stored descending with a shift sigma = (R - len) mod 4, which makes the
// A range and the B range of every tile share one 16-byte phase.
#pragma once
#include "bcf_kernels.cuh"
#include "bcf_tma.cuh"

namespace bcf {

constexpr int TMA_STAGES = 2;

template <int E, int U>
__host__ __device__ constexpr int stage_words() {
  return ((U * E + E + 8) + 3) / 4 * 4;  // T + cell-scan slack + shift, 16-B multiple
}
template <int E, int U, bool PAIRS>
__host__ __device__ constexpr size_t tma_smem_bytes() {
  return (size_t)TMA_STAGES * stage_words<E, U>() * sizeof(uint32_t) * (PAIRS ? 2 : 1);
}

struct TileMeta {
  long long c0;  // output global word of logical output index q
  int NA, NB, cnt, c, cout, qlo, qhi, desc;
};

__device__ __forceinline__ int align_up4(int x) { return (x + 3) & ~3; }
__device__ __forceinline__ int align_dn4(int x) { return x & ~3; }

// merge path with an initial bracket [lo, hi] (all lanes get the answer)
__device__ __forceinline__ long long merge_path_warp_global_bounded(const RunView& A, const RunView& B,
                                                                    long long D, long long lo, long long hi,
                                                                    int lane) {
  long long l2 = D - B.len;
  if (lo < l2) lo = l2;
  if (lo < 0) lo = 0;
  long long h2 = D < A.len ? D : A.len;
  if (hi > h2) hi = h2;
  while (hi > lo) {
    const long long cnt = hi - lo;
    const long long s = (cnt + 31) >> 5;
    const long long m = lo + (long long)(lane + 1) * s - 1;
    bool p = false;
    if (m < hi) {
      const uint32_t a = A.ld(m);
      const uint32_t b = B.ld(D - 1 - m);
      p = !(b < a);
    }
    const int c = __popc(__ballot_sync(FULL, p));
    const long long nlo = lo + (long long)c * s;
    long long nhi = lo + (long long)(c + 1) * s - 1;
    if (nhi > hi) nhi = hi;
    lo = nlo;
    hi = nhi;
  }
  return lo;
}

template <int E, int U, bool PAIRS>
__global__ void __launch_bounds__(U + 32) merge_pass_tma_kernel(MergeArgs args, long long tiles,
                                                                long long per_cta) {
  constexpr int T = U * E;
  constexpr int NW = U / W;
  constexpr int SW = stage_words<E, U>();
  constexpr int S = TMA_STAGES;
  static_assert(cgcd(W, E) == 1, "TMA staging needs rho = identity (E coprime with 32)");
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  __shared__ TileMeta meta[S];
  __shared__ __align__(8) uint64_t full_bar[S];
  __shared__ __align__(8) uint64_t empty_bar[S];
  __shared__ int s_org[NW + 1];

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & (W - 1);
  const long long t_begin = (long long)blockIdx.x * per_cta;
  long long t_end = t_begin + per_cta;
  if (t_end > tiles) t_end = tiles;
  const int m = (int)(t_end - t_begin);
  if (m <= 0) return;  // uniform over the CTA

  auto stage_k = [&](int s) { return smem_dyn + (size_t)s * SW * (PAIRS ? 2 : 1); };
  auto stage_v = [&](int s) { return smem_dyn + (size_t)s * SW * (PAIRS ? 2 : 1) + SW; };

  if (tid == 0) {
    for (int s = 0; s < S; ++s) {
      tma::mbar_init(&full_bar[s], 1);
      tma::mbar_init(&empty_bar[s], 1);
    }
  }
  __syncthreads();

  if (warp == NW) {
    // =========================== producer ===========================
    const uint32_t* __restrict__ srck = args.src_k;
    const uint32_t* __restrict__ srcv = args.src_v;
    uint32_t* __restrict__ dstk = args.dst_k;
    uint32_t* __restrict__ dstv = args.dst_v;
    const long long dst_phase = (long long)(((uintptr_t)dstk >> 2) & 3);
    long long prev_a1 = 0, prev_tb = -1;

    // bulk store of the outputs held in stage s (tile described by meta[s])
    auto store_out = [&](int s) {
      const TileMeta M = meta[s];
      uint32_t* sk = stage_k(s);
      uint32_t* sv = stage_v(s);
      const int w0 = M.cout + M.qlo, w1 = M.cout + M.qhi;  // stage words holding the tile
      const long long g0 = M.c0 - M.cout;                  // global word of stage word 0
      int ilo = align_up4(w0), ihi = align_dn4(w1);
      if (ihi <= ilo) ilo = ihi = w1;  // tiny tile: everything via lanes
      if (lane == 0 && ihi > ilo) {
        tma::bulk_s2g(dstk + g0 + ilo, sk + ilo, (uint32_t)(ihi - ilo) * 4u);
        if constexpr (PAIRS) tma::bulk_s2g(dstv + g0 + ilo, sv + ilo, (uint32_t)(ihi - ilo) * 4u);
        tma::bulk_commit();
      }
      // head words [w0, ilo) and tail words [ihi, w1): at most 3 + 3 (or 7)
      {
        const int nh = ilo - w0;
        int w = -1;
        if (lane < nh) w = w0 + lane;
        else if (lane >= 8 && lane - 8 < w1 - ihi) w = ihi + (lane - 8);
        if (w >= 0) {
          dstk[g0 + w] = sk[w];
          if constexpr (PAIRS) dstv[g0 + w] = sv[w];
        }
      }
      if (lane == 0) tma::bulk_wait_read_all();
      __syncwarp();
    };

    for (int i = 0; i < m; ++i) {
      const int s = i % S;
      const uint32_t u = (uint32_t)(i / S);
      const long long t = t_begin + i;
      long long j;
      const GroupDesc grp = group_of_tile(args, t, T, j);
      const long long lenG = grp.na + grp.nb;
      const long long D0 = j * T;
      const long long D1 = D0 + T < lenG ? D0 + T : lenG;
      RunView Av{srck + grp.a_off, grp.na, 0};
      RunView Bv{srck + grp.b_off, grp.nb, 1};
      long long a0;
      if (j == 0) a0 = 0;
      else if (prev_tb == grp.tile_begin) a0 = prev_a1;  // consecutive tile, same group
      else a0 = merge_path_warp_global(Av, Bv, D0, lane);
      long long a1;
      if (D1 == lenG) a1 = grp.na;
      else a1 = merge_path_warp_global_bounded(Av, Bv, D1, a0, a0 + (D1 - D0), lane);
      prev_a1 = a1;
      prev_tb = grp.tile_begin;
      const int cnt = (int)(D1 - D0);
      const int NA = (int)(a1 - a0);
      const int NB = cnt - NA;
      const long long b0 = D0 - a0;
      const long long oA = grp.a_off + a0;                     // A[a0 + q] at word oA + q
      const long long oB = grp.b_off + grp.nb - b0 - T;        // logical q (B part) at oB + q
      const int c = (int)(oA & 3);                             // src is 16-byte aligned
      TileMeta M;
      M.desc = grp.out_desc;
      M.c0 = M.desc ? grp.out_off + lenG - D0 - T : grp.out_off + D0;
      M.qlo = M.desc ? T - cnt : 0;
      M.qhi = M.desc ? T : cnt;
      M.cout = (int)((unsigned long long)(dst_phase + M.c0) & 3ull);
      M.NA = NA;
      M.NB = NB;
      M.cnt = cnt;
      M.c = c;

      if (i >= S) {
        tma::mbar_wait(&empty_bar[s], (u - 1) & 1);
        store_out(s);
      }
      if (lane == 0) meta[s] = M;

      // copy ranges in stage words: logical q lives at stage word c + q
      int a_hi = NA ? align_up4(c + NA) : 0;           // A: stage [0, a_hi)
      int b_lo = NB ? align_dn4(c + T - NB) : 0;       // B: stage [b_lo, b_hi)
      const int b_hi = NB ? align_up4(c + T) : 0;
      int ea0 = 0, ea1 = 0, eb0 = 0, eb1 = 0;          // edge words (stage indices)
      if (NA && NB && a_hi > b_lo) {
        ea1 = c + NA;
        a_hi = align_dn4(ea1);
        ea0 = a_hi;
        eb0 = c + T - NB;
        b_lo = align_up4(eb0);
        eb1 = b_lo;
      }
      uint32_t* sk = stage_k(s);
      uint32_t* sv = stage_v(s);
      if (lane == 0) {
        const uint32_t bytes = (uint32_t)(a_hi + (b_hi - b_lo)) * 4u * (PAIRS ? 2u : 1u);
        tma::mbar_expect_tx(&full_bar[s], bytes);
        if (a_hi > 0) {
          tma::bulk_g2s(sk, srck + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s]);
          if constexpr (PAIRS) tma::bulk_g2s(sv, srcv + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s]);
        }
        if (b_hi > b_lo) {
          tma::bulk_g2s(sk + b_lo, srck + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s]);
          if constexpr (PAIRS)
            tma::bulk_g2s(sv + b_lo, srcv + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s]);
        }
      }
      // misaligned edge words around the A/B boundary (generic loads/stores)
      {
        int w = -1;
        long long gw = 0;
        if (lane >= 1 && lane <= 3 && ea0 + lane - 1 < ea1) {
          w = ea0 + lane - 1;
          gw = oA + (w - c);
        } else if (lane >= 4 && lane <= 6 && eb0 + lane - 4 < eb1) {
          w = eb0 + lane - 4;
          gw = oB + (w - c);
        }
        if (w >= 0) {
          sk[w] = __ldg(srck + gw);
          if constexpr (PAIRS) sv[w] = __ldg(srcv + gw);
        }
      }
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(&full_bar[s]);
    }
    // drain: store the last min(S, m) tiles
    for (int i = (m > S ? m - S : 0); i < m; ++i) {
      const int s = i % S;
      tma::mbar_wait(&empty_bar[s], (uint32_t)(i / S) & 1);
      store_out(s);
    }
    if (lane == 0) tma::bulk_wait_all();
    return;
  }

  // ============================ consumers ============================
  const bool decode = args.decode_f32 != 0;
  for (int i = 0; i < m; ++i) {
    const int s = i % S;
    tma::mbar_wait(&full_bar[s], (uint32_t)(i / S) & 1);
    const TileMeta M = meta[s];
    uint32_t* sk = stage_k(s) + M.c;  // logical index -> sk[index]
    uint32_t* sv = stage_v(s) + M.c;
    const int NA = M.NA, NB = M.NB, cnt = M.cnt;
    uint32_t key[E], val[E];
    const int D = tid * E;
    const int Dw = warp * W * E;
    const int alpha = warp_origin_smem<E>(sk, 0, T, NA, NB, Dw, lane);
    if (lane == 0) s_org[warp] = alpha;
    if (tid == 0) s_org[NW] = NA;
    tma::named_bar_sync(1, U);
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
    if (decode) {
#pragma unroll
      for (int q = 0; q < E; ++q) key[q] = f32_decode(key[q]);
    }
    tma::named_bar_sync(1, U);  // every consumer has finished reading the stage
    uint32_t* ok = stage_k(s) + M.cout;
    uint32_t* ov = stage_v(s) + M.cout;
    if (M.desc) {
#pragma unroll
      for (int q = 0; q < E; ++q) {
        ok[T - E - D + q] = key[E - 1 - q];
        if constexpr (PAIRS) ov[T - E - D + q] = val[E - 1 - q];
      }
    } else {
#pragma unroll
      for (int q = 0; q < E; ++q) {
        ok[D + q] = key[q];
        if constexpr (PAIRS) ov[D + q] = val[q];
      }
    }
    tma::fence_proxy_async_smem();
    tma::named_bar_sync(1, U);
    if (tid == 0) tma::mbar_arrive(&empty_bar[s]);
  }
}

}  // namespace bcf
