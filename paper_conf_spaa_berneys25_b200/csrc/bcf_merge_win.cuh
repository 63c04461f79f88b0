// bcf_merge_win.cuh -- persistent CF merge pass with self-splitting tiles
// (keys only, E coprime with 32).
//
// A CTA (NW consumer warps + 1 producer warp) walks a contiguous chunk of
// output tiles.  Tile i starts at the merge-path point (a0, b0) -- known from
// the previous tile -- and the producer bulk-loads (TMA) a WINDOW of T keys
// of A from a0 and T keys of B from b0 into a 2-stage shared ring, laid out
// as the paper's rho(A u pi(B)) over a span of 2T (A at [0, WA), B reversed
// at [2T - WB, 2T); 2T is a multiple of wE, so every round set of §3.3 is
// unchanged).  The first T outputs only involve keys inside the windows, so
// the consumers find the tile's own end split a(T) in shared memory (warp 0,
// conflict-free 32-ary search) while the other warps compute their origins;
// warp 0 publishes the split through an mbarrier and the producer
// immediately bulk-loads the next tile's window.  The window data beyond the
// tile is re-read by the next tile from L2 (DRAM traffic stays ~8 B/key).
// The only global merge-path search left is the first boundary of a chunk
// that starts inside a merge group.
#pragma once
#include "bcf_merge_tma.cuh"

namespace bcf {

template <int E, int U>
__host__ __device__ constexpr int win_stage_words() {
  return ((2 * U * E + E + 8) + 3) / 4 * 4;  // 2T + cell-scan slack + shift
}
constexpr int WIN_STAGES = 2;
template <int E, int U>
__host__ __device__ constexpr size_t win_smem_bytes() {
  return (size_t)WIN_STAGES * win_stage_words<E, U>() * sizeof(uint32_t);
}

struct WinMeta {
  long long c0;       // output global word of logical output index q
  int WA, WB;         // window sizes (keys of A / B present)
  int cnt, c, cout, qlo, qhi, desc;
  int NA;             // tile's A count, written by the consumers
};

template <int E, int U>
__global__ void __launch_bounds__(U + 32) merge_pass_win_kernel(MergeArgs args, long long tiles,
                                                                long long per_cta) {
  constexpr int T = U * E;
  constexpr int T2 = 2 * T;
  constexpr int NW = U / W;
  constexpr int SW = win_stage_words<E, U>();
  constexpr int S = WIN_STAGES;
  static_assert(cgcd(W, E) == 1, "window staging needs rho = identity (E coprime with 32)");
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  __shared__ WinMeta meta[S];
  __shared__ __align__(8) uint64_t full_bar[S];
  __shared__ __align__(8) uint64_t empty_bar[S];
  __shared__ __align__(8) uint64_t split_bar[S];
  __shared__ int s_org[NW + 1];

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & (W - 1);
  const long long t_begin = (long long)blockIdx.x * per_cta;
  long long t_end = t_begin + per_cta;
  if (t_end > tiles) t_end = tiles;
  const int m = (int)(t_end - t_begin);
  if (m <= 0) return;
  auto stage = [&](int s) { return smem_dyn + (size_t)s * SW; };

  if (tid == 0) {
    for (int s = 0; s < S; ++s) {
      tma::mbar_init(&full_bar[s], 1);
      tma::mbar_init(&empty_bar[s], 1);
      tma::mbar_init(&split_bar[s], 1);
    }
  }
  __syncthreads();

  if (warp == NW) {
    // =========================== producer ===========================
    const uint32_t* __restrict__ src = args.src_k;
    const long long dst_phase = (long long)(((uintptr_t)args.dst_k >> 2) & 3);

    // window load of tile t starting at merge-path point a0 into stage s
    auto load_window = [&](int s, long long t, long long a0) {
      long long j;
      const GroupDesc grp = group_of_tile(args, t, T, j);
      const long long lenG = grp.na + grp.nb;
      const long long D0 = j * T;
      const long long b0 = D0 - a0;
      WinMeta M;
      const long long cnt = lenG - D0 < T ? lenG - D0 : T;
      M.cnt = (int)cnt;
      M.WA = (int)(grp.na - a0 < T ? grp.na - a0 : T);
      M.WB = (int)(grp.nb - b0 < T ? grp.nb - b0 : T);
      const long long oA = grp.a_off + a0;                  // A[a0 + q] at word oA + q
      const long long oB = grp.b_off + grp.nb - b0 - T2;    // logical q (B part) at oB + q
      const int c = (int)(oA & 3);
      M.c = c;
      M.desc = grp.out_desc;
      M.c0 = M.desc ? grp.out_off + lenG - D0 - T : grp.out_off + D0;
      M.qlo = M.desc ? T - M.cnt : 0;
      M.qhi = M.desc ? T : M.cnt;
      M.cout = (int)((unsigned long long)(dst_phase + M.c0) & 3ull);
      M.NA = 0;
      if (lane == 0) meta[s] = M;
      const int WA = M.WA, WB = M.WB;
      int a_hi = WA ? align_up4(c + WA) : 0;
      int b_lo = WB ? align_dn4(c + T2 - WB) : 0;
      const int b_hi = WB ? align_up4(c + T2) : 0;
      int ea0 = 0, ea1 = 0, eb0 = 0, eb1 = 0;
      if (WA && WB && a_hi > b_lo) {
        ea1 = c + WA;
        a_hi = align_dn4(ea1);
        ea0 = a_hi;
        eb0 = c + T2 - WB;
        b_lo = align_up4(eb0);
        eb1 = b_lo;
      }
      uint32_t* sk = stage(s);
      // edge words first (their loads overlap the bulk-copy issue)
      int w = -1;
      long long gw = 0;
      if (lane >= 1 && lane <= 3 && ea0 + lane - 1 < ea1) {
        w = ea0 + lane - 1;
        gw = oA + (w - c);
      } else if (lane >= 4 && lane <= 6 && eb0 + lane - 4 < eb1) {
        w = eb0 + lane - 4;
        gw = oB + (w - c);
      }
      const uint32_t ev = w >= 0 ? __ldg(src + gw) : 0u;
      if (lane == 0) {
        tma::mbar_expect_tx(&full_bar[s], (uint32_t)(a_hi + (b_hi - b_lo)) * 4u);
        if (a_hi > 0) tma::bulk_g2s(sk, src + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s]);
        if (b_hi > b_lo) tma::bulk_g2s(sk + b_lo, src + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s]);
      }
      if (w >= 0) sk[w] = ev;
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(&full_bar[s]);
      return grp.tile_begin;
    };

    // chunk start: the only global merge-path search
    long long a0;
    {
      long long j;
      const GroupDesc grp = group_of_tile(args, t_begin, T, j);
      const long long D0 = j * T;
      RunView Av{src + grp.a_off, grp.na, 0};
      RunView Bv{src + grp.b_off, grp.nb, 1};
      a0 = j == 0 ? 0 : merge_path_warp_global_bounded(Av, Bv, D0, 0, D0, lane);
    }
    if (lane == 0) BCF_TRACE_AT(0);
    long long tb = load_window(0, t_begin, a0);
    if (lane == 0) BCF_TRACE_AT(128 + 2);
    for (int i = 0; i < m; ++i) {
      const int s = i % S;
      const uint32_t u = (uint32_t)(i / S);
      // tile i's own end split, found by its consumers
      tma::mbar_wait(&split_bar[s], u & 1);
      if (lane == 0) BCF_TRACE_AT(128 + 4 * i + 1);
      const int NA = meta[s].NA;
      if (i + 1 < m) {
        long long j1;
        const GroupDesc g1 = group_of_tile(args, t_begin + i + 1, T, j1);
        const long long a_next = (g1.tile_begin == tb) ? a0 + NA : 0;
        const int s1 = (i + 1) % S;
        if (i >= 1) {
          // stage s1 held tile i-1: its consumers must have copied it out
          tma::mbar_wait(&empty_bar[s1], (uint32_t)((i - 1) / S) & 1);
          if (lane == 0) BCF_TRACE_AT(128 + 4 * (i + 1) + 3);
        }
        a0 = a_next;
        tb = load_window(s1, t_begin + i + 1, a0);
        if (lane == 0) BCF_TRACE_AT(128 + 4 * (i + 1) + 2);
      }
    }
    return;
  }

  // ============================ consumers ============================
  const bool decode = args.decode_f32 != 0;
  uint32_t dummy[E];
  for (int i = 0; i < m; ++i) {
    const int s = i % S;
    if (tid == 0) BCF_TRACE_AT(1 + 4 * i);
    tma::mbar_wait(&full_bar[s], (uint32_t)(i / S) & 1);
    if (tid == 0) BCF_TRACE_AT(2 + 4 * i);
    const WinMeta M = meta[s];
    uint32_t* sk = stage(s) + M.c;  // logical index -> sk[index]
    const int WA = M.WA, WB = M.WB, cnt = M.cnt;
    const int D = tid * E;
    const int Dw = warp * W * E;
    // warp 0: the tile's end split a(cnt) (its own origin is 0); other warps:
    // their origins a(Dw).  Window bounds are exact for every D <= cnt.
    const int probe = warp == 0 ? cnt : Dw;
    const int r = warp_origin_smem<E>(sk, 0, T2, WA, WB, probe, lane);
    const int alpha = warp == 0 ? 0 : r;
    if (lane == 0) s_org[warp] = alpha;
    if (warp == 0 && lane == 0) {
      s_org[NW] = r;
      meta[s].NA = r;
      tma::mbar_arrive(&split_bar[s]);  // release: the producer loads the next window
    }
    tma::named_bar_sync(1, U);
    // splits past the tile's last output are a(cnt) = NA (windows extend
    // beyond the tile, so they must be clamped explicitly)
    const int NA = s_org[NW];
    int a = lane_split_smem<E>(sk, 0, T2, WA, WB, Dw, alpha, lane, W, 5);
    if (D >= cnt) a = NA;
    int anext = __shfl_down_sync(FULL, a, 1);
    if (lane == W - 1) anext = (warp + 1) * W * E >= cnt ? NA : s_org[warp + 1];
    const int Dc = D < cnt ? D : cnt;
    const int Dn = D + E < cnt ? D + E : cnt;
    const int nA = anext - a;
    const int nB = (Dn - Dc) - nA;
    const int b = Dc - a;
    uint32_t key[E];
    if (cnt == T)
      dual_subsequence_gather<E, false, true>(sk, sk, 0, T2, a, b, nA, nB, key, dummy, PAD_KEY);
    else
      dual_subsequence_gather<E, false, false>(sk, sk, 0, T2, a, b, nA, nB, key, dummy, PAD_KEY);
    merge_registers<E, false>(key, dummy, a, nA, nB);
    if (decode) {
#pragma unroll
      for (int q = 0; q < E; ++q) key[q] = f32_decode(key[q]);
    }
    tma::named_bar_sync(1, U);  // every consumer has finished reading the stage
    uint32_t* ok = stage(s) + M.cout;
    if (M.desc) {
#pragma unroll
      for (int q = 0; q < E; ++q) ok[T - E - D + q] = key[E - 1 - q];
    } else {
#pragma unroll
      for (int q = 0; q < E; ++q) ok[D + q] = key[q];
    }
    tma::named_bar_sync(1, U);
    // copy-out: the tile's outputs sit at stage words [w0, w1), stage word w
    // belongs at global word g0 + w and both are 16-byte aligned for w = 0
    // (mod 4): vectorised conflict-free LDS.128 / coalesced STG.128, plus at
    // most 3 + 3 edge words.
    {
      const int w0 = M.cout + M.qlo, w1 = M.cout + M.qhi;
      int ilo = align_up4(w0), ihi = align_dn4(w1);
      if (ihi < ilo) ilo = ihi = w1;
      const uint32_t* sb = stage(s);
      uint32_t* gb = args.dst_k + (M.c0 - M.cout);
#pragma unroll
      for (int r = 0; r < (T + 4 * U - 1) / (4 * U) + 1; ++r) {
        const int v = ilo + 4 * (tid + r * U);
        if (v < ihi) *reinterpret_cast<uint4*>(gb + v) = *reinterpret_cast<const uint4*>(sb + v);
      }
      const int nh = ilo - w0;
      if (tid < nh) gb[w0 + tid] = sb[w0 + tid];
      else if (tid >= 32 && tid - 32 < w1 - ihi) gb[ihi + tid - 32] = sb[ihi + tid - 32];
    }
    tma::named_bar_sync(1, U);  // stage reads done: hand it back to the producer
    if (tid == 0) tma::mbar_arrive(&empty_bar[s]);
    if (tid == 0) BCF_TRACE_AT(3 + 4 * i);
  }
}

}  // namespace bcf
