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

#ifndef BCF_TMA_STAGES
#define BCF_TMA_STAGES 3
#endif
#ifndef BCF_TMA_MINB
#define BCF_TMA_MINB 1
#endif
// startup boundary search: 0 = producer only (sequential), 1 = every warp,
// 64-ary; 2 = every warp, 32-ary
#ifndef BCF_STARTUP
#define BCF_STARTUP 1
#endif
constexpr int TMA_STAGES = BCF_TMA_STAGES;

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

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// debug timeline: 256 slots per CTA (consumers at 1 + 4i, producer at 128 + 4i)
#define BCF_TRACE_AT(slot)                                                          \
  do {                                                                              \
    if (args.trace && args.npass <= 1 && (slot) < 256) args.trace[(size_t)blockIdx.x * 256 + (slot)] = gtimer(); \
  } while (0)

// tiles [t_begin, t_end) of this CTA: per_cta > 0 -> fixed chunks of per_cta
// tiles; per_cta == 0 -> the tiles spread evenly over the grid (chunks differ
// by at most one tile, so a grid of SMs x resident CTAs is load-balanced)
__device__ __forceinline__ void cta_tile_range(long long tiles, long long per_cta, long long& t_begin,
                                               long long& t_end) {
  const long long b = blockIdx.x;
  if (per_cta > 0) {
    t_begin = b * per_cta;
    t_end = t_begin + per_cta;
  } else {
    t_begin = b * tiles / gridDim.x;
    t_end = (b + 1) * tiles / gridDim.x;
  }
  if (t_end > tiles) t_end = tiles;
}

__device__ __forceinline__ int align_up4(int x) { return (x + 3) & ~3; }
__device__ __forceinline__ int align_dn4(int x) { return x & ~3; }

// merge path with an initial bracket [lo, hi] (all lanes get the answer):
// 64-ary search, every lane tests two candidates per round (4 independent
// loads in flight), so a bracket of one tile (<= 4096) takes 2 rounds of
// global-memory latency and a full run of 2^23 takes 4.
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
    const long long s = (cnt + 63) >> 6;  // probe stride, 64 probes
    const long long m0 = lo + (long long)(2 * lane + 1) * s - 1;
    const long long m1 = m0 + s;
    uint32_t a0 = 0, b0 = 0, a1 = 0, b1 = 0;
    if (m0 < hi) { a0 = A.ld(m0); b0 = B.ld(D - 1 - m0); }
    if (m1 < hi) { a1 = A.ld(m1); b1 = B.ld(D - 1 - m1); }
    const bool p0 = m0 < hi && !(b0 < a0);
    const bool p1 = m1 < hi && !(b1 < a1);
    const int c = __popc(__ballot_sync(FULL, p0)) + __popc(__ballot_sync(FULL, p1));
    const long long nlo = lo + (long long)c * s;
    long long nhi = lo + (long long)(c + 1) * s - 1;
    if (nhi > hi) nhi = hi;
    lo = nlo;
    hi = nhi;
  }
  return lo;
}

// Bracketed merge path that first tests 64 candidates around a guess (the
// proportional split of the remaining elements), spaced by s1 ~ sqrt(D)/16:
// for random keys a(D) deviates from the guess by O(sqrt(D)), so it lies
// inside the probed bracket (+-32 s1, about 8 standard deviations) and a
// second round at stride 1 (s1 <= 64) finishes the search: two rounds of
// global-memory latency.  Otherwise the 64-ary search continues on the
// reduced bracket.
__device__ __forceinline__ long long merge_path_warp_global_guess(const RunView& A, const RunView& B,
                                                                  long long D, long long lo, long long hi,
                                                                  long long guess, int lane) {
  long long l2 = D - B.len;
  if (lo < l2) lo = l2;
  if (lo < 0) lo = 0;
  long long h2 = D < A.len ? D : A.len;
  if (hi > h2) hi = h2;
  if (hi <= lo) return lo;
  long long s1 = (long long)sqrtf((float)(D < 1 ? 1 : D)) / 16;
  if (s1 < 1) s1 = 1;
  if (s1 > 64) s1 = 64;
  // probes m_i = L + (i+1) s1 - 1, i = 0..63 (lane tests i = 2 lane, 2 lane + 1)
  long long L = guess - 32 * s1;
  if (L > hi - 64 * s1) L = hi - 64 * s1;
  if (L < lo) L = lo;
  const long long m0 = L + (2 * lane + 1) * s1 - 1, m1 = m0 + s1;
  uint32_t a0 = 0, b0 = 0, a1 = 0, b1 = 0;
  if (m0 < hi) { a0 = A.ld(m0); b0 = B.ld(D - 1 - m0); }
  if (m1 < hi) { a1 = A.ld(m1); b1 = B.ld(D - 1 - m1); }
  const bool p0 = m0 < hi && !(b0 < a0);
  const bool p1 = m1 < hi && !(b1 < a1);
  const unsigned bal0 = __ballot_sync(FULL, p0), bal1 = __ballot_sync(FULL, p1);
  const int c = __popc(bal0) + __popc(bal1);  // Q true for the first c probes
  // answer in [L + c s1, L + (c+1) s1 - 1] when probe c exists and is false
  long long nlo = L + (long long)c * s1;
  long long nhi = L + (long long)(c + 1) * s1 - 1;
  if (nhi > hi) nhi = hi;
  if (c == 0) return L == lo ? (s1 == 1 ? lo : merge_path_warp_global_bounded(A, B, D, lo, L + s1 - 1, lane))
                             : merge_path_warp_global_bounded(A, B, D, lo, L + s1 - 1, lane);
  if (c == 64) return merge_path_warp_global_bounded(A, B, D, L + 64 * s1, hi, lane);
  if (s1 == 1 || nlo >= nhi) return nlo;
  return merge_path_warp_global_bounded(A, B, D, nlo, nhi, lane);
}

template <int E, int U, bool PAIRS>
__global__ void __launch_bounds__(U + 32, BCF_TMA_MINB) merge_pass_tma_kernel(MergeArgs args, long long tiles,
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
  __shared__ long long s_bnd[NW + 2];  // precomputed boundaries (see below)

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & (W - 1);
  long long t_begin, t_end;
  cta_tile_range(tiles, per_cta, t_begin, t_end);
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
  tma::pdl_wait();     // pass i reads what pass i-1 wrote (and overwrites what it read)
  tma::pdl_trigger();  // one persistent wave: the next pass may queue for our slots
  // Startup: the NW + 1 warps compute, in parallel, the merge-path
  // boundaries of the first tiles of the chunk (full-range 64-ary searches):
  // s_bnd[k] = a(start of tile k) for k < min(m, NW + 1), and
  // s_bnd[NW + 1] = a(end of the last tile) when m <= NW + 1.  The producer's
  // steady state then starts with no search on its critical path.
  const int npre = BCF_STARTUP == 0 ? 0 : (m < NW + 1 ? m : NW + 1);
  if (BCF_STARTUP != 0) {
    int k = warp;
    const bool last = (m <= NW + 1) && (warp == m % (NW + 1));  // spare warp: end of last tile
    if (k < npre || last) {
      const long long t = t_begin + (last ? m - 1 : k);
      long long j;
      const GroupDesc grp = group_of_tile(args, t, T, j);
      const long long lenG = grp.na + grp.nb;
      long long D = j * T;
      if (last) D = D + T < lenG ? D + T : lenG;
      RunView Av{args.src_k + grp.a_off, grp.na, 0};
      RunView Bv{args.src_k + grp.b_off, grp.nb, 1};
      long long a;
      if (D == 0) a = 0;
      else if (D == lenG) a = grp.na;
      else if (BCF_STARTUP == 2) a = merge_path_warp_global(Av, Bv, D, lane);
      else a = merge_path_warp_global_bounded(Av, Bv, D, 0, D, lane);
      if (lane == 0) s_bnd[last ? NW + 1 : k] = a;
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
      if (lane == 0) {
        if (ihi > ilo) {
          tma::bulk_s2g(dstk + g0 + ilo, sk + ilo, (uint32_t)(ihi - ilo) * 4u);
          if constexpr (PAIRS) tma::bulk_s2g(dstv + g0 + ilo, sv + ilo, (uint32_t)(ihi - ilo) * 4u);
        }
        tma::bulk_commit();  // one group per tile (possibly empty): wait_group counts tiles
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
      __syncwarp();
    };

    // Split of tile t (merge-path boundaries a0, a1 and the tile descriptor);
    // consecutive tiles of the chunk reuse the previous boundary, so the
    // search for a1 is bracketed to a range of T (3 rounds of 32 probes).
    struct Split {
      TileMeta M;
      long long oA, oB;
      int ea0, ea1, eb0, eb1, a_hi, b_lo, b_hi;  // copy plan (stage words)
      int ew;                                    // this lane's edge word (-1: none)
      uint32_t ek, ev;                           // its value (loaded early)
    };
    auto split_of = [&](long long t) {
      long long j;
      const GroupDesc grp = group_of_tile(args, t, T, j);
      const long long lenG = grp.na + grp.nb;
      const long long D0 = j * T;
      const long long D1 = D0 + T < lenG ? D0 + T : lenG;
      RunView Av{srck + grp.a_off, grp.na, 0};
      RunView Bv{srck + grp.b_off, grp.nb, 1};
      const int i = (int)(t - t_begin);
      long long a0;
      if (i < npre) a0 = s_bnd[i];
      else if (j == 0) a0 = 0;
      else if (prev_tb == grp.tile_begin) a0 = prev_a1;  // consecutive tile, same group
      else a0 = merge_path_warp_global_bounded(Av, Bv, D0, 0, D0, lane);
      long long a1;
      if (D1 == lenG) a1 = grp.na;
      else if (i + 1 < npre) a1 = s_bnd[i + 1];
      else if (npre > 0 && i + 1 == m && m <= NW + 1) a1 = s_bnd[NW + 1];
      else {
        const long long rest = lenG - D0;
        const long long guess = a0 + (long long)((double)(D1 - D0) * (double)(grp.na - a0) / (double)rest);
        a1 = merge_path_warp_global_guess(Av, Bv, D1, a0, a0 + (D1 - D0), guess, lane);
      }
      prev_a1 = a1;
      prev_tb = grp.tile_begin;
      // L2 prefetch of the next tile's A and B ranges: they hold the probes
      // of the next split search and the next bulk loads
      if (lane == 0 && D1 < lenG) {
        const long long b1 = D1 - a1;
        const long long ahi = a1 + T < grp.na ? a1 + T : grp.na;
        const long long bhi = b1 + T < grp.nb ? b1 + T : grp.nb;
        if (ahi > a1) {
          const long long w0 = (grp.a_off + a1) & ~3ll, w1 = (grp.a_off + ahi + 3) & ~3ll;
          tma::bulk_prefetch_l2(srck + w0, (uint32_t)(w1 - w0) * 4u);
        }
        if (bhi > b1) {  // B[y] at b_off + nb-1-y: y in [b1, bhi) -> [b_off+nb-bhi, b_off+nb-b1)
          const long long w0 = (grp.b_off + grp.nb - bhi) & ~3ll, w1 = (grp.b_off + grp.nb - b1 + 3) & ~3ll;
          tma::bulk_prefetch_l2(srck + w0, (uint32_t)(w1 - w0) * 4u);
        }
      }
      Split sp;
      const int cnt = (int)(D1 - D0);
      const long long b0 = D0 - a0;
      sp.oA = grp.a_off + a0;                     // A[a0 + q] at word oA + q
      sp.oB = grp.b_off + grp.nb - b0 - T;        // logical q (B part) at oB + q
      sp.M.desc = grp.out_desc;
      sp.M.c0 = sp.M.desc ? grp.out_off + lenG - D0 - T : grp.out_off + D0;
      sp.M.qlo = sp.M.desc ? T - cnt : 0;
      sp.M.qhi = sp.M.desc ? T : cnt;
      sp.M.cout = (int)((unsigned long long)(dst_phase + sp.M.c0) & 3ull);
      const int NA = (int)(a1 - a0), NB = cnt - NA, c = (int)(sp.oA & 3);  // src 16-B aligned
      sp.M.NA = NA;
      sp.M.NB = NB;
      sp.M.cnt = cnt;
      sp.M.c = c;
      // copy plan: logical q lives at stage word c + q; A -> [0, a_hi),
      // B -> [b_lo, b_hi); a 16-byte chunk shared by A's tail and B's head is
      // filled word by word (edge words)
      sp.a_hi = NA ? align_up4(c + NA) : 0;
      sp.b_lo = NB ? align_dn4(c + T - NB) : 0;
      sp.b_hi = NB ? align_up4(c + T) : 0;
      sp.ea0 = sp.ea1 = sp.eb0 = sp.eb1 = 0;
      if (NA && NB && sp.a_hi > sp.b_lo) {
        sp.ea1 = c + NA;
        sp.a_hi = align_dn4(sp.ea1);
        sp.ea0 = sp.a_hi;
        sp.eb0 = c + T - NB;
        sp.b_lo = align_up4(sp.eb0);
        sp.eb1 = sp.b_lo;
      }
      // issue the edge-word loads now; they are consumed by load_tile later
      sp.ew = -1;
      sp.ek = sp.ev = 0;
      long long gw = 0;
      if (lane >= 1 && lane <= 3 && sp.ea0 + lane - 1 < sp.ea1) {
        sp.ew = sp.ea0 + lane - 1;
        gw = sp.oA + (sp.ew - c);
      } else if (lane >= 4 && lane <= 6 && sp.eb0 + lane - 4 < sp.eb1) {
        sp.ew = sp.eb0 + lane - 4;
        gw = sp.oB + (sp.ew - c);
      }
      if (sp.ew >= 0) {
        sp.ek = __ldg(srck + gw);
        if constexpr (PAIRS) sp.ev = __ldg(srcv + gw);
      }
      return sp;
    };

    // bulk loads of tile i (described by sp) into stage s
    auto load_tile = [&](int s, const Split& sp) {
      if (lane == 0) meta[s] = sp.M;
      uint32_t* sk = stage_k(s);
      uint32_t* sv = stage_v(s);
      const int c = sp.M.c;
      if (lane == 0) {
        const uint32_t bytes = (uint32_t)(sp.a_hi + (sp.b_hi - sp.b_lo)) * 4u * (PAIRS ? 2u : 1u);
        tma::mbar_expect_tx(&full_bar[s], bytes);
        if (sp.a_hi > 0) {
          tma::bulk_g2s(sk, srck + (sp.oA - c), (uint32_t)sp.a_hi * 4u, &full_bar[s]);
          if constexpr (PAIRS) tma::bulk_g2s(sv, srcv + (sp.oA - c), (uint32_t)sp.a_hi * 4u, &full_bar[s]);
        }
        if (sp.b_hi > sp.b_lo) {
          const uint32_t nb = (uint32_t)(sp.b_hi - sp.b_lo) * 4u;
          tma::bulk_g2s(sk + sp.b_lo, srck + (sp.oB + sp.b_lo - c), nb, &full_bar[s]);
          if constexpr (PAIRS) tma::bulk_g2s(sv + sp.b_lo, srcv + (sp.oB + sp.b_lo - c), nb, &full_bar[s]);
        }
      }
      if (sp.ew >= 0) {
        sk[sp.ew] = sp.ek;
        if constexpr (PAIRS) sv[sp.ew] = sp.ev;
      }
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(&full_bar[s]);
    };

    // Schedule per tile i (S = 3 stages):
    //   wait for tile i-2's outputs, issue its bulk store (no read wait);
    //   wait until tile i-3's store has read its stage (issued one step ago);
    //   load tile i into that stage; search the split of tile i+1 while the
    //   consumers compute tile i-1.
    if (lane == 0) BCF_TRACE_AT(0);
    if (lane == 0) BCF_TRACE_AT(128);
    Split cur = split_of(t_begin);
    if (lane == 0) BCF_TRACE_AT(129);
    for (int i = 0; i < m; ++i) {
      const int s = i % S;
      if (i >= 2) {
        const int k = i - 2;
        tma::mbar_wait(&empty_bar[k % S], (uint32_t)(k / S) & 1);
        if (lane == 0) BCF_TRACE_AT(128 + 4 * i + 3);
        store_out(k % S);  // issue + commit, no read wait
      }
      if (i >= S) {
        // stage s held tile i-3, whose store was committed one step ago
        if (lane == 0) tma::bulk_wait_read_1();
        __syncwarp();
      }
      load_tile(s, cur);
      if (lane == 0) BCF_TRACE_AT(128 + 4 * i + 2);
      if (i + 1 < m) cur = split_of(t_begin + i + 1);
      if (lane == 0) BCF_TRACE_AT(128 + 4 * (i + 1) + 1);
    }
    // drain: the last two tiles
    for (int k = (m >= 2 ? m - 2 : 0); k < m; ++k) {
      tma::mbar_wait(&empty_bar[k % S], (uint32_t)(k / S) & 1);
      store_out(k % S);
    }
    if (lane == 0) tma::bulk_wait_all();
    return;
  }

  // ============================ consumers ============================
  const bool decode = args.decode_f32 != 0;
  for (int i = 0; i < m; ++i) {
    const int s = i % S;
    if (tid == 0) BCF_TRACE_AT(1 + 4 * i);
    tma::mbar_wait(&full_bar[s], (uint32_t)(i / S) & 1);
    if (tid == 0) BCF_TRACE_AT(2 + 4 * i);
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
    if (tid == 0) BCF_TRACE_AT(3 + 4 * i);
  }
}

}  // namespace bcf
