// bcf_merge_win.cuh -- persistent CF merge pass with self-splitting,
// variable-size tiles (keys only, E coprime with 32).
//
// A CTA (NW consumer warps + 1 producer warp) walks a contiguous range of the
// pass's output (the tiles [t_begin, t_end) of T = U*E outputs each) as a
// sequence of SUBTILES of at most T outputs.  Subtile i starts at the
// merge-path point (a0, b0) -- known from subtile i-1 -- and the producer
// bulk-loads (TMA) a window of WA keys of A from a0 and WB keys of B from b0
// into a 2-stage shared ring.  The stage is the paper's rho(A u pi(B)) over a
// span of S2 = T + T/4 words (A at [0, WA), B reversed at [S2 - WB, S2); S2
// is a multiple of wE, so every round set of §3.3 is unchanged), with
// WA + WB = S2: the split of the span between A and B is predicted from the
// previous subtile's A share.  The first outputs of the merge only involve
// keys inside the windows, so the consumers find the subtile's own end split
// in shared memory (warp 0, conflict-free k-ary search), and if the merge path
// leaves a window before T outputs (a badly predicted or skewed split) the
// subtile simply ends there, at a multiple of 4 outputs (the rare path).  Warp 0
// publishes (count, split) through an mbarrier and the producer immediately
// bulk-loads the next window.  A span of 1.25 T instead of 2 T (one window
// of T keys per run) keeps five CTAs resident per SM for (E, u) = (31, 128).
// The only global merge-path search left is the first boundary of a CTA's
// range when it starts inside a merge group.
#pragma once
#include "bcf_merge_tma.cuh"

namespace bcf {

// L2 hints of the window kernel's bulk copies (A/B builds): bit 0 = window
// loads evict_first (the pass's input is dead once read), bit 1 = output
// stores evict_last (the next pass reads them)
#ifndef BCF_L2_HINTS
#define BCF_L2_HINTS 1  // measured: loads evict_first +1.4 % at 2^24 (35.8 vs 36.7 us per pass)
#endif
// L2 prefetch distance beyond each window, in quarters of a tile (A/B builds)
#ifndef BCF_WIN_PF
#define BCF_WIN_PF 0  // measured: no prefetch is best (2^24: 35.4 vs 35.9 us per pass; 2^28: 0.796 vs 0.782 of HBM)
#endif

#ifndef BCF_WIN_Q
#define BCF_WIN_Q 1  // span S2 = T + Q * T/4 (Q = 4: two full windows, never exhausted)
#endif

template <int E, int U>
__host__ __device__ constexpr int win_span() {
  return U * E + BCF_WIN_Q * (U / 4) * E;  // U/4 is a multiple of w: S2 = 0 (mod wE)
}
template <int E, int U>
__host__ __device__ constexpr int win_stage_words() {
  // span + cell-scan slack + shift; with rho != identity the slack probes of
  // logical words past the span land anywhere in the next rho partition
  constexpr int d = cgcd(W, E);
  constexpr int slack = (d > 1 && W * E / d > E + 8) ? W * E / d : E + 8;
  return ((win_span<E, U>() + slack) + 3) / 4 * 4;
}
#ifndef BCF_WIN_STAGES
#define BCF_WIN_STAGES 2
#endif
constexpr int WIN_STAGES = BCF_WIN_STAGES;
template <int E, int U, bool PAIRS = false>
__host__ __device__ constexpr size_t win_smem_bytes() {
  return (size_t)WIN_STAGES * win_stage_words<E, U>() * sizeof(uint32_t) * (PAIRS ? 2 : 1);
}

// progress words of a multi-pass launch: per-CTA flags at [0, MULTI_COUNTERS_AT),
// then one completed-CTA counter per pass
constexpr int MULTI_COUNTERS_AT = 1536;

struct WinMeta {
  long long c0;       // output global word of logical output index q
  int WA, WB;         // window sizes (keys of A / B present)
  int cmax;           // outputs wanted (<= T); the consumers may end earlier
  int fin;            // bit 0: A window holds every A key the subtile can need; bit 1: B
  int c, cout, desc, exit;
  int NA, cnt;        // the subtile's A count and output count (consumers)
};

// Number of leading elements of a sorted window for which pred holds
// (pred true on a prefix).  Warp-cooperative 32-ary search; the probes of one
// round are at an odd stride, i.e. distinct banks for consecutive storage (or
// reversed consecutive storage) under rho = identity.
template <class P>
__device__ __forceinline__ int warp_prefix_count(int n, P pred, int lane) {
  int lo = 0, hi = n;
  while (hi > lo) {
    const int s = (((hi - lo) + 31) >> 5) | 1;
    const int m = lo + (lane + 1) * s - 1;
    const bool p = m < hi && pred(m);
    const int c = __popc(__ballot_sync(FULL, p));
    const int nlo = lo + c * s;
    int nhi = lo + (c + 1) * s - 1;
    if (nhi > hi) nhi = hi;
    lo = nlo;
    hi = nhi;
    if (s == 1) break;
  }
  return lo;
}

// The same count for a window stored through rho (E sharing factors with w):
// key(m) reads logical word l0 + sgn * m.  Probes at stride f E (f odd) form a
// round set (Lemma 1 / Cor. 3), so every round reads 32 distinct banks; the
// last <= E candidates are consecutive words, read in two halves split at the
// rho partition boundary (consecutive words inside one partition are
// consecutive banks modulo its rotation).
template <int E, class P>
__device__ __forceinline__ int warp_prefix_count_rho(int n, P pred, int l0, int sgn, int lane) {
  int lo = 0, hi = n;
  while (hi - lo > E) {
    const int need = ((hi - lo) + 31) >> 5;
    const int f = ((need + E - 1) / E) | 1;
    const int st = f * E;
    const int m = lo + (lane + 1) * st - 1;
    const bool p = m < hi && pred(m);
    const int c = __popc(__ballot_sync(FULL, p));
    const int nlo = lo + c * st;
    int nhi = lo + (c + 1) * st - 1;
    if (nhi > hi) nhi = hi;
    lo = nlo;
    hi = nhi;
  }
  const int m = lo + lane;
  const bool act = m < hi;
  // logical word of candidate m, and the partition boundary after lo's word
  const int w0 = l0 + sgn * lo;
  const int pend = sgn > 0 ? rho_partition_end<E>(w0) : rho_partition_end<E>(w0) - W * E / cgcd(W, E);
  const int wm = l0 + sgn * m;
  const bool first = sgn > 0 ? wm < pend : wm >= pend;
  bool p = false;
  if (act && first) p = pred(m);
  __syncwarp();
  if (act && !first) p = pred(m);
  return lo + __popc(__ballot_sync(FULL, p));
}

// resident CTAs per SM the kernel is built for (5 at u = 128)
template <int U, bool PAIRS = false, int E = 0>
__host__ __device__ constexpr int win_min_blocks() {
  // pairs: twice the stage bytes and a value + tag register per key
#ifndef BCF_WIN_PAIRS_MINB256
#define BCF_WIN_PAIRS_MINB256 3  // 3 CTAs/SM at (11, 256): <= 75 registers (the pass loop of the multi-pass mode had raised ptxas's choice to 95, 2 CTAs/SM)
#endif
  if (PAIRS) return U <= 128 ? 3 : (U <= 256 ? (E <= 13 ? BCF_WIN_PAIRS_MINB256 : 2) : 1);
  return WIN_STAGES > 2 ? (U <= 128 ? 3 : 1) : (U <= 128 ? 5 : (U <= 256 ? 2 : 1));
}

// MULTI: the multi-pass instantiation (MergeArgs::npass passes in one launch);
// the one-pass kernel does not carry its machinery (registers: (11, 256)
// pairs 95 -> 72, (11, 256) keys 88 -> 64)
template <int E, int U, bool PAIRS = false, bool MULTI = false>
__global__ void __launch_bounds__(U + 32, win_min_blocks<U, PAIRS, E>()) merge_pass_win_kernel(MergeArgs args, long long tiles,
                                                                long long per_cta) {
  constexpr int T = U * E;
  constexpr int S2 = win_span<E, U>();
  constexpr int NW = U / W;
  constexpr int SW = win_stage_words<E, U>();
  constexpr int S = WIN_STAGES;
  // E sharing factors with w (d > 1, rho != identity, §3.2): the
  // producer stages windows in rho's physical order with 4-byte cp.async
  // (bulk copies cannot rotate 4-byte words inside a partition), the
  // consumers copy the outputs out with LSU loads / stores
  constexpr bool RHO = cgcd(W, E) > 1;
  static_assert(S2 % (W * E) == 0 && S2 % 4 == 0 && S2 > T, "span must be a multiple of wE");
  extern __shared__ __align__(16) uint32_t smem_dyn[];
  __shared__ WinMeta meta[S];
  __shared__ __align__(8) uint64_t full_bar[S];
  __shared__ __align__(8) uint64_t empty_bar[S];
  __shared__ __align__(8) uint64_t split_bar[S];
  __shared__ int s_org[NW + 2];

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & (W - 1);
  long long t_begin, t_end;
  cta_tile_range(tiles, per_cta, t_begin, t_end);
  if (t_end <= t_begin) return;
  // multi-pass mode: passes p = 0..npass-1 of a sort in this one launch
  // (MergeArgs::npass); a CTA keeps its tile range in every pass
  // (MULTI instantiation: the multi-pass machinery, used when args.npass > 1)
  const bool multi = MULTI && args.npass > 1;
  const int npass = multi ? args.npass : 1;
  auto pass_args = [&](int p) {
    MergeArgs a = args;
    if (multi) {
      const bool last = p == npass - 1;
      a.src_k = args.buf_k[p & 1];
      a.src_v = args.buf_v[p & 1];
      a.dst_k = last ? args.dst_k : args.buf_k[(p + 1) & 1];
      a.dst_v = last ? args.dst_v : args.buf_v[(p + 1) & 1];
      a.R = args.R << p;
      a.log2_tpg = args.log2_tpg + p;
      a.decode_f32 = last ? args.decode_f32 : 0;
    }
    return a;
  };
  // stage s: SW key words, then (pairs) SW value words at the same offsets
  auto stage = [&](int s) { return smem_dyn + (size_t)s * SW * (PAIRS ? 2 : 1); };
  auto stage_v = [&](int s) { return smem_dyn + (size_t)s * SW * (PAIRS ? 2 : 1) + SW; };

  if (tid == 0) {
    for (int s = 0; s < S; ++s) {
      tma::mbar_init(&full_bar[s], RHO ? 32 : 1);
      tma::mbar_init(&empty_bar[s], 1);
      tma::mbar_init(&split_bar[s], 1);
    }
  }
  __syncthreads();
  tma::pdl_wait();     // pass i reads what pass i-1 wrote (and overwrites what it read)
  tma::pdl_trigger();  // one persistent wave: the next pass may queue for our slots

  if (warp == NW) {
    // =========================== producer ===========================
    // the CTA owning tile t (inverse of cta_tile_range with per_cta = 0)
    auto cta_of_tile = [&](long long t) {
      const long long G = gridDim.x;
      long long c = (t * G) / tiles;
      while (c + 1 < G && ((c + 1) * tiles) / G <= t) ++c;
      while (c > 0 && (c * tiles) / G > t) --c;
      return c;
    };
    int i = 0;  // ring index over every subtile and pass-end marker of the launch
    for (int p = 0; p < npass; ++p) {
    const MergeArgs args = pass_args(p);  // shadows the launch arguments inside the pass
    if (p > 0) {
      // pass p reads the groups of pass p-1 that its tiles fall in: wait until
      // every CTA covering them has published pass p-1, then order the bulk
      // copies below after those acquires
      const int l = args.log2_tpg;
      const long long gb = (t_begin >> l) << l;
      long long ge = (((t_end - 1) >> l) + 1) << l;
      if (ge > tiles) ge = tiles;
      const long long c_lo = cta_of_tile(gb), c_hi = cta_of_tile(ge - 1);
      if (lane == 0 && args.trace) args.trace[(size_t)blockIdx.x * 256 + 4 * p] = gtimer();
      if (c_hi - c_lo + 1 >= (long long)gridDim.x) {
        // every CTA: the pass counter (one word) instead of G flags
        const unsigned* cnt = args.progress + MULTI_COUNTERS_AT + (p - 1);
        while (tma::ld_acquire_gpu(cnt) < gridDim.x) __nanosleep(200);
      } else {
        for (;;) {
          bool ok = true;
          for (long long c = c_lo + lane; c <= c_hi; c += W)
            ok = ok && tma::ld_acquire_gpu(args.progress + c) >= (unsigned)p;
          if (__all_sync(FULL, ok)) break;
          __nanosleep(200);
        }
      }
      __syncwarp();
      tma::fence_proxy_async_global();
      if (lane == 0 && args.trace) args.trace[(size_t)blockIdx.x * 256 + 4 * p + 1] = gtimer();
    }
    const uint32_t* __restrict__ src = args.src_k;
    // B runs (table mode, bcf_merge_u32): a separate base, stored descending
    const uint32_t* __restrict__ srcB = args.src_kb ? args.src_kb : args.src_k;
    const uint32_t* __restrict__ srcv = args.src_v;
    const uint32_t* __restrict__ srcvB = args.src_vb ? args.src_vb : args.src_v;
    const long long dst_phase = (long long)(((uintptr_t)args.dst_k >> 2) & 3);

    // current segment: the part of one merge group inside this CTA's range
    long long j0;
    GroupDesc grp = group_of_tile(args, t_begin, T, j0);
    auto seg_end = [&](const GroupDesc& g, long long tile0) {
      const long long lenG = g.na + g.nb;
      long long te = g.tile_begin + (lenG + T - 1) / T;
      if (te > t_end) te = t_end;
      long long De = (te - g.tile_begin) * T;
      return De < lenG ? De : lenG;
    };
    long long Dend = seg_end(grp, t_begin);
    long long D0 = j0 * T;
    long long a0;
    {
      RunView Av{src + grp.a_off, grp.na, 0, multi ? 1 : 0};
      RunView Bv{srcB + grp.b_off, grp.nb, 1, multi ? 1 : 0};
      const long long lenG = grp.na + grp.nb;
      const long long guess = lenG > 0 ? (long long)((double)D0 * (double)grp.na / (double)lenG) : 0;
      a0 = j0 == 0 ? 0 : merge_path_warp_global_guess(Av, Bv, D0, 0, D0, guess, lane);
    }
    // predicted A share of the next subtile (fraction of outputs, x 2^16)
    int shareA = (grp.na + grp.nb) > 0 ? (int)((grp.na << 16) / (grp.na + grp.nb)) : 32768;

    // subtile window of the current (grp, D0, a0) into stage s
    auto load_window = [&](int s) {
      const long long lenG = grp.na + grp.nb;
      const long long b0 = D0 - a0;
      WinMeta M;
      const int cmax = (int)(Dend - D0 < T ? Dend - D0 : T);
      const long long remA = grp.na - a0, remB = grp.nb - b0;
      const int needA = (int)(remA < cmax ? remA : cmax);
      const int needB = (int)(remB < cmax ? remB : cmax);
      int WA, WB;
      if (needA + needB <= S2) {
        WA = needA;
        WB = needB;
      } else {
        // predicted A count + half the slack, clamped so that both windows fit
        int pa = (int)(((long long)shareA * cmax) >> 16) + (S2 - cmax) / 2;
        const int lo = S2 - needB, hi = needA;
        pa = pa < lo ? lo : (pa > hi ? hi : pa);
        WA = pa;
        WB = S2 - pa;
      }
      M.WA = WA;
      M.WB = WB;
      M.cmax = cmax;
      M.fin = (WA == needA ? 1 : 0) | (WB == needB ? 2 : 0);
      M.exit = 0;
      const long long oA = grp.a_off + a0;                  // A[a0 + q] at word oA + q
      const long long oB = grp.b_off + grp.nb - b0 - S2;    // logical q (B part) at oB + q
      const int c = RHO ? 0 : (int)(oA & 3);
      M.c = c;
      M.desc = grp.out_desc;
      M.c0 = M.desc ? grp.out_off + lenG - D0 - T : grp.out_off + D0;
      M.cout = RHO ? 0 : (int)((unsigned long long)(dst_phase + M.c0) & 3ull);
      M.NA = 0;
      M.cnt = 0;
      if (lane == 0) meta[s] = M;
      auto prefetch_next = [&]() {
        if constexpr (BCF_WIN_PF == 0) return;
        // L2 prefetch of the keys the next window will need beyond this one
        // (both runs are consumed sequentially): the next window's loads,
        // issued one subtile later, then hit L2 instead of DRAM
        constexpr long long PF = (BCF_WIN_PF * T / 4 + 3) & ~3;
        const long long pa0 = (oA + WA + 3) & ~3ll;                  // A: ascending words
        long long pa1 = grp.a_off + grp.na;
        if (pa1 > pa0 + PF) pa1 = pa0 + PF;
        pa1 &= ~3ll;
        if (pa1 > pa0) tma::bulk_prefetch_l2(src + pa0, (uint32_t)(pa1 - pa0) * 4u);
        long long pb1 = (grp.b_off + grp.nb - b0 - WB) & ~3ll;      // B: descending words
        long long pb0 = grp.b_off;
        if (pb0 < pb1 - PF) pb0 = pb1 - PF;
        pb0 = (pb0 + 3) & ~3ll;
        if (pb1 > pb0) tma::bulk_prefetch_l2(srcB + pb0, (uint32_t)(pb1 - pb0) * 4u);
      };
      if constexpr (RHO) {
        // staged in PHYSICAL order: slot p (32 consecutive slots per warp
        // instruction, conflict-free writes) receives logical word
        // q = rho^-1(p): A from src[oA + q] (q < WA), B from srcB[oB + q]
        // (q >= S2 - WB = WA); the reads stay inside one or two rotated
        // partitions (coalesced)
        __syncwarp();  // meta[s] written before any lane's copies land
        uint32_t* sk = stage(s);
        for (int p = lane; p < S2; p += W) {
          const int q = rho_inv<E>(p);
          if (q >= WA && q < S2 - WB) continue;  // the gap between the windows (never read)
          const uint32_t* g = q < WA ? src + oA + q : srcB + oB + q;
          tma::cp_async4(sk + p, g);
          if constexpr (PAIRS) tma::cp_async4(stage_v(s) + p, (q < WA ? srcv + oA : srcvB + oB) + q);
        }
        if (lane == 0) {
          prefetch_next();
          tma::cp_async_wait_all();          // lane 0: its copies, then a release arrive (meta)
          tma::mbar_arrive(&full_bar[s]);
        } else {
          tma::cp_async_mbar_arrive_noinc(&full_bar[s]);  // when this lane's copies have landed
        }
        __syncwarp();
        return;
      }
      int a_hi = WA ? align_up4(c + WA) : 0;
      int b_lo = WB ? align_dn4(c + S2 - WB) : 0;
      const int b_hi = WB ? align_up4(c + S2) : 0;
      int ea0 = 0, ea1 = 0, eb0 = 0, eb1 = 0;
      if (WA && WB && a_hi > b_lo) {
        ea1 = c + WA;
        a_hi = align_dn4(ea1);
        ea0 = a_hi;
        eb0 = c + S2 - WB;
        b_lo = align_up4(eb0);
        eb1 = b_lo;
      }
      // the aligned A range must not run past A's last word (a caller's
      // array, bcf_merge_u32): its last <= 3 words then come from the edge
      // lanes instead (after the overlap split, which clips A the same way)
      if (WA && (long long)a_hi > grp.a_off + grp.na - (oA - c)) {
        ea1 = c + WA;
        a_hi = align_dn4(ea1);
        ea0 = a_hi;
      }
      uint32_t* sk = stage(s);
      // edge words first (their loads overlap the bulk-copy issue)
      int w = -1;
      long long gw = 0;
      const uint32_t* __restrict__ esrc = lane >= 4 ? srcB : src;
      const uint32_t* __restrict__ esrcv = lane >= 4 ? srcvB : srcv;
      if (lane >= 1 && lane <= 3 && ea0 + lane - 1 < ea1) {
        w = ea0 + lane - 1;
        gw = oA + (w - c);
      } else if (lane >= 4 && lane <= 6 && eb0 + lane - 4 < eb1) {
        w = eb0 + lane - 4;
        gw = oB + (w - c);
      }
      if (lane == 0) {
        tma::mbar_expect_tx(&full_bar[s], (uint32_t)(a_hi + (b_hi - b_lo)) * 4u * (PAIRS ? 2u : 1u));
        if constexpr ((BCF_L2_HINTS & 1) != 0) {
          const uint64_t pol = tma::policy_evict_first();
          if (a_hi > 0) tma::bulk_g2s_hint(sk, src + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s], pol);
          if (b_hi > b_lo)
            tma::bulk_g2s_hint(sk + b_lo, srcB + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s], pol);
        } else {
          if (a_hi > 0) tma::bulk_g2s(sk, src + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s]);
          if (b_hi > b_lo) tma::bulk_g2s(sk + b_lo, srcB + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s]);
        }
        if constexpr (PAIRS) {
          uint32_t* sv = stage_v(s);
          if constexpr ((BCF_L2_HINTS & 1) != 0) {
            const uint64_t pol = tma::policy_evict_first();
            if (a_hi > 0) tma::bulk_g2s_hint(sv, srcv + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s], pol);
            if (b_hi > b_lo)
              tma::bulk_g2s_hint(sv + b_lo, srcvB + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s], pol);
          } else {
            if (a_hi > 0) tma::bulk_g2s(sv, srcv + (oA - c), (uint32_t)a_hi * 4u, &full_bar[s]);
            if (b_hi > b_lo)
              tma::bulk_g2s(sv + b_lo, srcvB + (oB + b_lo - c), (uint32_t)(b_hi - b_lo) * 4u, &full_bar[s]);
          }
        }
        prefetch_next();
      }
      uint32_t ev = 0u, evv = 0u;
      if (w >= 0) {
        ev = multi ? ld_cg(esrc + gw) : __ldg(esrc + gw);
        if constexpr (PAIRS) evv = multi ? ld_cg(esrcv + gw) : __ldg(esrcv + gw);
      }
      // lane 0 stores the <= 6 edge words itself, then release-arrives: the
      // stores precede the arrive in one thread's program order (a lane-l
      // store ordered only through __syncwarp is invisible to racecheck)
#pragma unroll
      for (int l = 1; l <= 6; ++l) {
        const int wl = __shfl_sync(FULL, w, l);
        const uint32_t kl = __shfl_sync(FULL, ev, l);
        const uint32_t vl = PAIRS ? __shfl_sync(FULL, evv, l) : 0u;
        if (lane == 0 && wl >= 0) {
          sk[wl] = kl;
          if constexpr (PAIRS) stage_v(s)[wl] = vl;
        }
      }
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(&full_bar[s]);
    };
    auto post_exit = [&](int s) {
      if (lane == 0) meta[s].exit = 1;
      __syncwarp();
      if (RHO || lane == 0) tma::mbar_arrive(&full_bar[s]);  // RHO: 32 arrivals per phase
      __syncwarp();
    };

    if (lane == 0) BCF_TRACE_AT(0);
    if (lane == 0 && args.trace) {
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      args.trace[(size_t)blockIdx.x * 256 + 255] = smid + 1;
    }
    // bulk store (TMA) of the outputs the consumers staged in stage s (the
    // 16-byte aligned middle; warp 0 of the consumers writes the <= 7 + 3
    // edge words).  Issued and waited on by lane 0 (bulk groups are per thread).
    auto store_out = [&](int s) {
      if constexpr (RHO) return;  // the consumers copy the outputs out
      const WinMeta M = meta[s];
      const int qlo = M.desc ? T - M.cnt : 0, qhi = M.desc ? T : M.cnt;
      const int w0 = M.cout + qlo, w1 = M.cout + qhi;
      int ilo = align_up4(w0), ihi = align_dn4(w1);
      if (lane == 0) {
        if (ihi > ilo) {
          if constexpr ((BCF_L2_HINTS & 2) != 0)
            tma::bulk_s2g_hint(args.dst_k + (M.c0 - M.cout) + ilo, stage(s) + ilo, (uint32_t)(ihi - ilo) * 4u,
                               tma::policy_evict_last());
          else
            tma::bulk_s2g(args.dst_k + (M.c0 - M.cout) + ilo, stage(s) + ilo, (uint32_t)(ihi - ilo) * 4u);
          if constexpr (PAIRS)
            tma::bulk_s2g(args.dst_v + (M.c0 - M.cout) + ilo, stage_v(s) + ilo, (uint32_t)(ihi - ilo) * 4u);
        }
        tma::bulk_commit();
      }
    };

    const int i0 = i;
    load_window(i % S);
    if (lane == 0) BCF_TRACE_AT(128 + 2);
    for (;; ++i) {
      const int s = i % S;
      const int s1 = (i + 1) % S;      // stage of the next window
      const int sp = (i + S - 1) % S;  // stage of subtile i-1 (= s1 for 2 stages)
      if (i >= i0 + 1) {
        // subtile i-1's outputs are staged in sp: stream them out while the
        // consumers search subtile i's split
        tma::mbar_wait(&empty_bar[sp], (uint32_t)((i - 1) / S) & 1);
        if (lane == 0 && i < 6) BCF_TRACE_AT(128 + 4 * (i + 1) + 3);
        store_out(sp);
      }
      // subtile i's own end split, found by its consumers
      tma::mbar_wait(&split_bar[s], (uint32_t)(i / S) & 1);
      if (lane == 0 && i < 7) BCF_TRACE_AT(128 + 4 * i + 1);
      const int NA = meta[s].NA, cnt = meta[s].cnt;
      if (cnt > 0) shareA = (int)(((long long)NA << 16) / cnt);
      D0 += cnt;
      a0 += NA;
      bool more = true;
      if (D0 >= Dend) {
        // segment done: the next one starts a new merge group at its first tile
        const long long tn = grp.tile_begin + (Dend + T - 1) / T;
        if (tn >= t_end) {
          more = false;
        } else {
          grp = group_of_tile(args, tn, T, j0);
          Dend = seg_end(grp, tn);
          D0 = 0;
          a0 = 0;
          shareA = (grp.na + grp.nb) > 0 ? (int)((grp.na << 16) / (grp.na + grp.nb)) : 32768;
        }
      }
      if (!more) {
        post_exit(s1);
        // the last subtile: stream its outputs, then drain every bulk store
        tma::mbar_wait(&empty_bar[s], (uint32_t)(i / S) & 1);
        store_out(s);
        if (lane == 0) tma::bulk_wait_all();
        __syncwarp();
        if (multi) {
          // the consumers acknowledge the pass-end marker on its split and
          // empty barriers (every barrier of a stage stays in phase), then
          // this CTA's outputs of pass p are published
          tma::mbar_wait(&split_bar[s1], (uint32_t)((i + 1) / S) & 1);
          tma::mbar_wait(&empty_bar[s1], (uint32_t)((i + 1) / S) & 1);
          if (lane == 0) {
            tma::fence_proxy_async_global();
            __threadfence();
            tma::st_release_gpu(args.progress + blockIdx.x, (unsigned)(p + 1));
            atomicAdd(args.progress + MULTI_COUNTERS_AT + p, 1u);  // pass counter (after the fence)
            if (args.trace) args.trace[(size_t)blockIdx.x * 256 + 4 * p + 2] = gtimer();
          }
          __syncwarp();
        }
        i += 2;  // the last subtile and the marker
        break;
      }
      // stage s1's last store (subtile i+1-S) has read it: with 2 stages that
      // is the store just issued, with more stages an older one
      if (lane == 0) {
        if constexpr (S == 2) tma::bulk_wait_read_all();
        else tma::bulk_wait_read_1();
      }
      __syncwarp();
      load_window(s1);
      if (lane == 0 && i < 6) BCF_TRACE_AT(128 + 4 * (i + 1) + 2);
    }
    }  // passes
    return;
  }

  // ============================ consumers ============================
  uint32_t val[E];  // values (pairs); unused for keys
  int i = 0;
  for (int p = 0; p < npass; ++p) {
  const MergeArgs args = pass_args(p);
  const bool decode = args.decode_f32 != 0;
  for (;; ++i) {
    const int s = i % S;
    if (tid == 0 && i < 31) BCF_TRACE_AT(1 + 4 * i);
    tma::mbar_wait(&full_bar[s], (uint32_t)(i / S) & 1);
    if (tid == 0 && i < 31) BCF_TRACE_AT(2 + 4 * i);
    const WinMeta M = meta[s];
    if (M.exit) {
      if (multi && tid == 0) {
        tma::mbar_arrive(&split_bar[s]);
        tma::mbar_arrive(&empty_bar[s]);
      }
      ++i;
      break;
    }
    uint32_t* sk = stage(s) + M.c;  // logical index -> sk[index]
    uint32_t* sv = stage_v(s) + M.c;
    const int WA = M.WA, WB = M.WB, cmax = M.cmax;
    const int D = tid * E;
    const int Dw = warp * W * E;
    // warp 0: the subtile's end split a(cmax) (its own origin is 0); other
    // warps: their origins a(Dw).  The window path equals the merge path as
    // long as neither window is exhausted early.
    const int probe = warp == 0 ? cmax : Dw;
    int r = warp_origin_smem<E>(sk, 0, S2, WA, WB, probe, lane);
    const int alpha = warp == 0 ? 0 : r;
    if (lane == 0) s_org[warp] = alpha;
    if (warp == 0) {
      int cnt = cmax;
      if (!(M.fin & 1) && r == WA) {
        // A window exhausted at D_A = WA + #{B[y] < A[WA-1]} (ties go to A)
        const uint32_t v = lds<E>(sk, WA - 1);
        int nb;
        if constexpr (RHO)
          nb = warp_prefix_count_rho<E>(WB, [&](int y) { return lds<E>(sk, S2 - 1 - y) < v; }, S2 - 1, -1, lane);
        else
          nb = warp_prefix_count(WB, [&](int y) { return sk[S2 - 1 - y] < v; }, lane);
        cnt = WA + nb;
      } else if (!(M.fin & 2) && cmax - r == WB) {
        // B window exhausted at D_B = WB + #{A[x] <= B[WB-1]}
        const uint32_t v = lds<E>(sk, S2 - WB);
        int na;
        if constexpr (RHO)
          na = warp_prefix_count_rho<E>(WA, [&](int x) { return !(v < lds<E>(sk, x)); }, 0, 1, lane);
        else
          na = warp_prefix_count(WA, [&](int x) { return !(v < sk[x]); }, lane);
        cnt = WB + na;
      }
      if (cnt < cmax) {
        // end on a multiple of 4 outputs (16-byte phase of the next windows)
        cnt &= ~3;
        r = warp_origin_smem<E>(sk, 0, S2, WA, WB, cnt, lane);
      }
      if (lane == 0) {
        s_org[NW] = r;
        s_org[NW + 1] = cnt;
        meta[s].NA = r;
        meta[s].cnt = cnt;
        tma::mbar_arrive(&split_bar[s]);  // release: the producer loads the next window
      }
    }
    tma::named_bar_sync(1, U);
    if (tid == 0 && i < 30) BCF_TRACE_AT(161 + 3 * i);
    // splits past the subtile's last output are a(cnt) = NA (windows extend
    // beyond it, so they must be clamped explicitly)
    const int NA = s_org[NW];
    const int cnt = s_org[NW + 1];
    int a = lane_split_smem<E>(sk, 0, S2, WA, WB, Dw, alpha, lane, W, 5);
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
      dual_subsequence_gather<E, PAIRS, true>(sk, PAIRS ? sv : sk, 0, S2, a, b, nA, nB, key, val, PAD_KEY);
    else
      dual_subsequence_gather<E, PAIRS, false>(sk, PAIRS ? sv : sk, 0, S2, a, b, nA, nB, key, val, PAD_KEY);
    merge_registers<E, PAIRS>(key, val, a, nA, nB);
    if (decode) {
#pragma unroll
      for (int q = 0; q < E; ++q) key[q] = f32_decode(key[q]);
    }
    tma::named_bar_sync(1, U);  // every consumer has finished reading the stage
    if (tid == 0 && i < 30) BCF_TRACE_AT(160 + 3 * i);
    uint32_t* ok = stage(s) + M.cout;
    uint32_t* ov = stage_v(s) + M.cout;
    // round m of the staging writes logical D + m (or its mirror): a round
    // set, conflict-free through rho (identity for E coprime with w)
    if (M.desc) {
#pragma unroll
      for (int q = 0; q < E; ++q) {
        ok[rho<E>(T - E - D + q)] = key[E - 1 - q];
        if constexpr (PAIRS) ov[rho<E>(T - E - D + q)] = val[E - 1 - q];
      }
    } else {
#pragma unroll
      for (int q = 0; q < E; ++q) {
        ok[rho<E>(D + q)] = key[q];
        if constexpr (PAIRS) ov[rho<E>(D + q)] = val[q];
      }
    }
    if constexpr (RHO) {
      // LSU copy-out: physical slot P (consecutive per warp, conflict-free)
      // holds logical output w = rho^-1(P), bound for global word c0 + w
      tma::named_bar_sync(1, U);
      const int qlo = M.desc ? T - cnt : 0;
      const int qhi = M.desc ? T : cnt;
      uint32_t* __restrict__ gk = args.dst_k + M.c0;
      uint32_t* __restrict__ gv = PAIRS ? args.dst_v + M.c0 : nullptr;
#pragma unroll
      for (int r = 0; r < E; ++r) {
        const int P = tid + r * U;
        const int w = rho_inv<E>(P);
        if (w >= qlo && w < qhi) {
          gk[w] = ok[P];
          if constexpr (PAIRS) gv[w] = ov[P];
        }
      }
      tma::named_bar_sync(1, U);  // every consumer has read the stage
      if (tid == 0) tma::mbar_arrive(&empty_bar[s]);
      continue;
    }
    tma::fence_proxy_async_smem();  // the producer's bulk store reads these words
    tma::named_bar_sync(1, U);
    if (tid == 0 && i < 31) BCF_TRACE_AT(4 + 4 * i);
    // the producer streams the 16-byte aligned middle of the outputs (stage
    // word w belongs at global word g0 + w, both aligned for w = 0 mod 4);
    // warp 0 writes the head/tail edge words, then hands the stage back
    if (warp == 0) {
      const int qlo = M.desc ? T - cnt : 0;
      const int qhi = M.desc ? T : cnt;
      const int w0 = M.cout + qlo, w1 = M.cout + qhi;
      int ilo = align_up4(w0), ihi = align_dn4(w1);
      if (ihi <= ilo) ilo = ihi = w1;
      const uint32_t* sb = stage(s);
      uint32_t* gb = args.dst_k + (M.c0 - M.cout);
      const int nh = ilo - w0, nt = w1 - ihi;  // <= 7, <= 3
      int ew = -1;
      if (lane < nh) ew = w0 + lane;
      else if (lane >= 8 && lane - 8 < nt) ew = ihi + lane - 8;
      if (ew >= 0) {
        gb[ew] = sb[ew];
        if constexpr (PAIRS) args.dst_v[(M.c0 - M.cout) + ew] = stage_v(s)[ew];
      }
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(&empty_bar[s]);
    }
    if (tid == 0 && i < 31) BCF_TRACE_AT(3 + 4 * i);
  }
  }  // passes
}

}  // namespace bcf
