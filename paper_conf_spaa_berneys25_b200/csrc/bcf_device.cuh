// bcf_device.cuh -- device primitives of the bank-conflict-free (CF) mergesort.
//
// Notation follows Berney & Sitchinava, "Eliminating Bank Conflicts in GPU
// Mergesort", SPAA'25: w = 32 banks / warp lanes, E items per
// thread, d = GCD(w, E), u = U threads per block, tile T = U*E.
//
// Shared-memory tile layout (Alg. 1 line 2; §3.3):
//     logical index k:  A[x] at k = x,  B[y] at k = T-1-y  (pi: B reversed)
//     physical index  = rho(k): partitions of P = wE/d elements rotated right
//                       by (partition mod d)            (§3.2)
// With this layout every shared-memory instruction below touches, per warp,
// a "round set" {k = j (mod E)} of one window of wE logical indices (or
// consecutive physical words), which is a complete residue system mod w
// (Lemma 1 / Corollary 3) -> zero bank conflicts for every input.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bcf {

constexpr int W = 32;  // banks = warp width on sm_100a (32 banks x 4 B)
constexpr unsigned FULL = 0xffffffffu;

__host__ __device__ constexpr int cgcd(int a, int b) { return b == 0 ? a : cgcd(b, a % b); }
__host__ __device__ constexpr int clog2(int x) { return x <= 1 ? 0 : 1 + clog2(x >> 1); }
__host__ __device__ constexpr int cpow2ceil(int x) { return x <= 1 ? 1 : 2 * cpow2ceil((x + 1) >> 1); }
__host__ __device__ constexpr bool is_pow2(int x) { return x > 0 && (x & (x - 1)) == 0; }

// ---------------------------------------------------------------------------
// rho: logical -> physical shared-memory word.
// Periodic with period wE (d partitions), so banks depend on k mod wE only.
// ---------------------------------------------------------------------------
template <int E>
__device__ __forceinline__ int rho(int k_) {
  constexpr int d = cgcd(W, E);
  if constexpr (d == 1) {
    return k_;
  } else {
    constexpr unsigned P = W * E / d;
    const unsigned k = (unsigned)k_;
    const unsigned l = k / P;                     // constant divisor
    if constexpr (is_pow2(P)) {
      return (int)((k & ~(P - 1)) | ((k + (l % d)) & (P - 1)));
    } else {
      const unsigned x = k - l * P;
      unsigned y = x + (l % d);
      y = y >= P ? y - P : y;
      return (int)(l * P + y);
    }
  }
}

template <int E>
__device__ __forceinline__ int rho_inv(int p_) {
  constexpr int d = cgcd(W, E);
  if constexpr (d == 1) {
    return p_;
  } else {
    constexpr unsigned P = W * E / d;
    const unsigned p = (unsigned)p_;
    const unsigned l = p / P;
    if constexpr (is_pow2(P)) {
      return (int)((p & ~(P - 1)) | ((p + P - (l % d)) & (P - 1)));
    } else {
      const unsigned y = p - l * P;
      const unsigned x = y >= (l % d) ? y - (l % d) : y + P - (l % d);
      return (int)(l * P + x);
    }
  }
}

// shared-memory load of logical index k (through rho)
template <int E>
__device__ __forceinline__ uint32_t lds(const uint32_t* __restrict__ sk, int k) {
  return sk[rho<E>(k)];
}

// First logical index of the next rho-partition after k (for splitting a run
// of consecutive probes at the partition wrap).
template <int E>
__device__ __forceinline__ int rho_partition_end(int k) {
  constexpr int d = cgcd(W, E);
  constexpr unsigned P = W * E / d;
  return (int)(((unsigned)k / P + 1) * P);
}

// ---------------------------------------------------------------------------
// Run views in global memory.  A sorted run of `len` keys is stored either
// ascending or descending (the CF pipeline stores every odd run of a pass
// descending, so that the tile stage writes B reversed = pi(B) with unit-stride
// reads).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t ld_cg(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

struct RunView {
  const uint32_t* base;
  long long len;
  int desc;      // 1: element y lives at base[len-1-y]
  int coherent = 0;  // 1: L2-coherent loads (data written earlier in the same launch by other CTAs)
  __device__ __forceinline__ long long addr(long long y) const { return desc ? (len - 1 - y) : y; }
  __device__ __forceinline__ uint32_t ld(long long y) const {
    return coherent ? ld_cg(base + addr(y)) : __ldg(base + addr(y));
  }
};

// ---------------------------------------------------------------------------
// Merge path (Green et al. [24]): number of A elements among the
// first D outputs of the stable merge of A and B (ties to A).  Warp-cooperative
// 32-ary search over global memory: each round every lane tests one candidate
// (2 independent loads), a ballot keeps the monotone prefix.  Returns the same
// value to all lanes.
// ---------------------------------------------------------------------------
__device__ __forceinline__ long long merge_path_warp_global(const RunView& A, const RunView& B,
                                                            long long D, int lane) {
  long long lo = D - B.len;
  if (lo < 0) lo = 0;
  long long hi = D < A.len ? D : A.len;
  // invariant: answer in [lo, hi]; Q(m) := a(D) >= m+1 := !(B[D-1-m] < A[m])
  while (hi > lo) {
    const long long cnt = hi - lo;
    const long long s = (cnt + 31) >> 5;  // probe stride
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
    if (s == 1) break;  // every candidate was tested: lo == answer
  }
  return lo;
}

// ---------------------------------------------------------------------------
// Conflict-free warp-origin search in shared memory.
// Returns a(D) for the merge group in smem (A[x] at logical base+x, B[y] at
// base+S2-1-y, S2 = group size, a multiple of wE).
// Probe stride s = fE with f odd: the 32 probes of a round are a round set of
// a window (mod wE), hence conflict-free under rho.  The last <= E consecutive
// probes are split at the rho-partition wrap.
// ---------------------------------------------------------------------------
template <int E>
__device__ __forceinline__ int warp_origin_smem(const uint32_t* __restrict__ sk, int base, int S2,
                                                int NA, int NB, int D, int lane) {
  if (D > NA + NB) D = NA + NB;  // a(D) = NA past the end (ragged tile)
  // A[x] at logical base+x; B[y] at base+S2-1-y, so B[D-1-m] at base+S2-D+m
  const int bofs = base + S2 - D;
  int lo = D - NB;
  if (lo < 0) lo = 0;
  int hi = D < NA ? D : NA;
  if constexpr (cgcd(W, E) == 1) {
    // rho = identity: any odd stride puts the 32 probes of one load in 32
    // distinct banks, so each round tests 64 candidates (two loads per side):
    // a range of 64^2 = 4096 takes two rounds
    while (hi > lo) {
      const int cnt = hi - lo;
      const int s = ((cnt + 63) >> 6) | 1;
      // candidate i at lo + (i+1)s - 1: load 1 tests i = lane, load 2 i = lane + 32
      const int q0 = lo + (lane + 1) * s - 1;       // candidate lane
      const int q1 = lo + (lane + 33) * s - 1;      // candidate lane + 32
      bool p0 = false, p1 = false;
      if (q0 < hi) p0 = !(sk[bofs + q0] < sk[base + q0]);
      if (q1 < hi) p1 = !(sk[bofs + q1] < sk[base + q1]);
      const unsigned b0 = __ballot_sync(FULL, p0), b1 = __ballot_sync(FULL, p1);
      const int c = __popc(b0) + __popc(b1);  // monotone: the first c candidates hold
      const int nlo = lo + c * s;
      int nhi = lo + (c + 1) * s - 1;
      if (nhi > hi) nhi = hi;
      lo = nlo;
      hi = nhi;
      if (s == 1) break;
    }
    return lo;
  }
  while (hi - lo > E) {
    const int cnt = hi - lo;
    // stride s = f*E with f odd and 32*s >= cnt: the 32 probes are = const
    // (mod E) and pairwise distinct mod wE -> a round set of a window.
    const int need = (cnt + 31) >> 5;
    int f = (need + E - 1) / E;
    f |= 1;
    const int s = f * E;
    const int m = lo + (lane + 1) * s - 1;
    bool p = false;
    if (m < hi) {
      const uint32_t a = lds<E>(sk, base + m);
      const uint32_t b = lds<E>(sk, bofs + m);
      p = !(b < a);
    }
    const int c = __popc(__ballot_sync(FULL, p));
    const int nlo = lo + c * s;
    int nhi = lo + (c + 1) * s - 1;
    if (nhi > hi) nhi = hi;
    lo = nlo;
    hi = nhi;
  }
  // final: candidates m = lo + lane, lane < hi - lo (<= E)
  const int m = lo + lane;
  const bool act = m < hi;
  uint32_t a = 0, b = 0;
  constexpr int d = cgcd(W, E);
  if constexpr (d == 1) {
    if (act) {
      a = sk[base + m];
      b = sk[bofs + m];
    }
  } else {
    const int aend = rho_partition_end<E>(base + lo);
    const int bend = rho_partition_end<E>(bofs + lo);
    if (act && base + m < aend) a = sk[rho<E>(base + m)];
    __syncwarp();
    if (act && base + m >= aend) a = sk[rho<E>(base + m)];
    __syncwarp();
    if (act && bofs + m < bend) b = sk[rho<E>(bofs + m)];
    __syncwarp();
    if (act && bofs + m >= bend) b = sk[rho<E>(bofs + m)];
  }
  const bool p = act && !(b < a);
  return lo + __popc(__ballot_sync(FULL, p));
}

// ---------------------------------------------------------------------------
// Conflict-free per-lane split search.
// The lanes [wb, wb+WL) of a warp form one "window": their diagonals are
// Dw + l'E (l' = lane - wb), the window's merge-path origin is alpha (so
// beta = Dw - alpha).  A[x] at logical base+x, B[y] at logical base+S2-1-y
// where S2 is the size of the merge group's tile/group (multiple of wE).
// Returns a(Dw + l'E) for the calling lane.
//   (2) corners: lane l' holds A[alpha+(l'+1)E-1] and B[beta+l'E] (stride E);
//       coarse cell M = max{m <= l' : Q(alpha+mE)} by shuffle bisection;
//   (3) cell scan: round j reads A[alpha+ME+j] and B[beta+(l'-M)E-1-j].
// ---------------------------------------------------------------------------
template <int E>
__device__ __forceinline__ int lane_split_smem(const uint32_t* __restrict__ sk, int base, int S2,
                                               int NA, int NB, int Dw, int alpha, int lane, int WL,
                                               int nit) {
  const int wb = lane & ~(WL - 1);
  const int lp = lane - wb;
  const int beta = Dw - alpha;
  const int D = Dw + lp * E;
  // (2) corners (stride E: a round set)
  const int ia = alpha + (lp + 1) * E - 1;
  const int ib = beta + lp * E;
  const uint32_t cA = ia < NA ? lds<E>(sk, base + ia) : 0u;
  const uint32_t cB = ib < NB ? lds<E>(sk, base + S2 - 1 - ib) : 0u;
  // coarse cell: largest m in [0, lp] with Q(alpha + mE), built bit by bit
  // (lanes of the window hold the corners; two shuffles per step).
  //   Q(m) = A-corner m-1 exists (m <= mA) and (B-corner lp-m is past B's end
  //          (lp - m >= kB) or !(B corner < A corner))
  const int mA = (NA - alpha) / E;
  const int kB = NB - beta > 0 ? (NB - beta + E - 1) / E : 0;
  int M = 0;
#pragma unroll
  for (int it = 0; it < 5; ++it) {
    const int st = 16 >> it;
    if (st < WL) {  // warp-uniform
      const int cnd = M + st;
      const bool inr = cnd <= lp;
      const uint32_t a = __shfl_sync(FULL, cA, wb + (inr ? cnd - 1 : 0));
      const uint32_t b = __shfl_sync(FULL, cB, wb + (inr ? lp - cnd : 0));
      const bool q = inr && cnd <= mA && (lp - cnd >= kB || !(b < a));
      M = q ? cnd : M;
    }
  }
  (void)nit;
  // (3) cell scan: round j tests Q(ac + j + 1) reading A[ac+j] and B[D-ac-1-j]
  const int ac = alpha + M * E;  // a(D) in [ac, ac+E]
  const int jA = (NA < D ? NA : D) - ac;   // j < jA: A[ac+j] exists and ac+j+1 <= D
  const int jB = D - ac - NB;              // j >= jB: B[D-ac-1-j] exists
  const int pa0 = base + ac;               // logical index of A[ac + j] = pa0 + j
  const int pb0 = base + S2 - D + ac;      // logical index of B[D-ac-1-j] = pb0 + j
  // Every probe is issued (indices outside [jB, jA) stay in the same round set,
  // so they cannot conflict; the tile buffer has E words of slack past its
  // end); the comparison bits are collected in a mask and the predicate is
  // true below jB, monotone on [jB, jA), false from jA on.
  uint32_t tm = 0;
#pragma unroll
  for (int j = 0; j < E; ++j) {
    const uint32_t ka = lds<E>(sk, pa0 + j);
    const uint32_t kb = lds<E>(sk, pb0 + j);
    tm |= (kb < ka) ? 0u : (1u << j);
  }
  // (past the end of the merge, D > NA + NB, jB exceeds jA: clamp)
  const int jAc = jA < 0 ? 0 : (jA > E ? E : jA);
  const int jBc = jB < 0 ? 0 : (jB > jAc ? jAc : jB);
  const uint32_t range = ((1u << jAc) - 1u) & ~((1u << jBc) - 1u);
  const int cnt = jBc + __popc(tm & range);
  return ac + cnt;
}

// ---------------------------------------------------------------------------
// Alg. 1 DUAL-SUBSEQUENCE-GATHER.  Thread with A offset a,
// B offset b (in its merge group), |A_i| = nA, |B_i| = nB (nA+nB <= E; fewer
// only in a ragged tile: those rounds read nothing and hold a pad).
// k = a mod E; round j reads A_i[(j-k) mod E] if that index < nA, else
// B_i[(k-j-1) mod E]; both at logical base + idx, B reversed behind A.
// After the gather, items[] is a circular bitonic sequence starting at k.
// ---------------------------------------------------------------------------
// rounds J.. of the gather for rho = identity (keys only): shared byte
// address = (A or B base, + E words when the round wraps) + 4J, the round
// index folded into the load's immediate offset (one select, one predicated
// add and the load per round)
template <int J, int E, bool FULL_TILE>
__device__ __forceinline__ void gather_rounds(uint32_t (&key)[E], uint32_t sA, uint32_t sB, uint32_t wmask,
                                              uint32_t maskA, int k, int nB, uint32_t pad) {
  if constexpr (J < E) {
    const bool wrap = (wmask >> J) & 1u;
    const bool isA = (maskA >> J) & 1u;
    uint32_t p = isA ? sA : sB;
    if (wrap) p += 4u * E;
    if constexpr (FULL_TILE) {
      asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(key[J]) : "r"(p), "n"(4 * J));
    } else {
      const int ia = wrap ? J + E - k : J - k;
      uint32_t v = pad;
      if (isA || (E - 1 - ia) < nB) asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(p), "n"(4 * J));
      key[J] = v;
    }
    gather_rounds<J + 1, E, FULL_TILE>(key, sA, sB, wmask, maskA, k, nB, pad);
  }
}

template <int E, bool PAIRS, bool FULL_TILE>
__device__ __forceinline__ void dual_subsequence_gather(const uint32_t* __restrict__ sk,
                                                        const uint32_t* __restrict__ sv, int base,
                                                        int S2, int a, int b, int nA, int nB,
                                                        uint32_t (&key)[E], uint32_t (&val)[E],
                                                        uint32_t pad) {
  const int k = a % E;
  // round j: ia = (j - k) mod E; A_i[ia] at logical base+a+ia, else
  // B_i[E-1-ia] at base+S2-1-(b+E-1-ia) = base+S2-b-E+ia.  Rounds reading A
  // form the circular range [k, k+nA): bit j of maskA.
  const int offA = base + a - k;
  const int offB = base + S2 - b - E - k;
  const uint32_t m0 = (1u << nA) - 1u;
  const uint32_t maskA = ((m0 << k) | (m0 >> (E - k))) & ((1u << E) - 1u);
  if constexpr (cgcd(W, E) == 1 && !PAIRS) {
    // rho = identity: select one of two shared-memory base pointers per
    // round and fold the round index into the load's immediate offset
    const uint32_t sA = (uint32_t)__cvta_generic_to_shared(sk) + 4u * (uint32_t)offA;
    const uint32_t sB = (uint32_t)__cvta_generic_to_shared(sk) + 4u * (uint32_t)offB;
    gather_rounds<0, E, FULL_TILE>(key, sA, sB, (1u << k) - 1u, maskA, k, nB, pad);
    return;
  }
  const int bAn = offA, bAw = offA + E, bBn = offB, bBw = offB + E;
#pragma unroll
  for (int j = 0; j < E; ++j) {
    const bool wrap = j < k;
    const bool isA = (maskA >> j) & 1u;
    const int idx = (wrap ? (isA ? bAw : bBw) : (isA ? bAn : bBn)) + j;
    bool ok = true;
    if constexpr (!FULL_TILE) {
      const int ia = wrap ? j + E - k : j - k;
      ok = isA || (E - 1 - ia) < nB;
    }
    if (ok) {
      key[j] = lds<E>(sk, idx);
      if constexpr (PAIRS) val[j] = lds<E>(sv, idx);
    } else {
      key[j] = pad;
      if constexpr (PAIRS) val[j] = 0;
    }
  }
}

// ---------------------------------------------------------------------------
// Compare-exchange helpers.  Keys-only: plain min/max (equal keys are equal
// bit patterns, so order among them is unobservable).  Pairs: lexicographic
// (key, tag) where tag is the element's rank in the stable order of the two
// inputs -- a strict total order, so any sorting network yields the stable
// result.
// ---------------------------------------------------------------------------
// Pipe balancing for keys-only compare-exchanges.  min/max run on the ALU
// pipe (64 lanes/clk/SM, the block sort's bound: ALU pipe ~87 % busy), the
// FMA pipe is nearly idle.  max(a, b) = a + b - min(a, b) (exact mod 2^32)
// as two IMADs puts the max on the FMA pipe; the multiplier is read from
// constant memory so ptxas cannot fold the IMAD back into an ALU IADD3.
// Networks use this form for 2 of every 3 compare-exchanges (ALU and FMA
// pipes then carry 4/3 instructions each per exchange instead of 2 + 0).
static __constant__ uint32_t c_one = 1u;

__device__ __forceinline__ uint32_t imad_u32(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  return r;
}

// which compare-exchanges take the FMA form (A/B builds: BCF_FMA_MOD = m puts
// the max of (m-1) of every m exchanges on the FMA pipe, 0 = none;
// BCF_LANE_FMA_MOD likewise for the cross-lane half-cleaner selects)
#ifndef BCF_FMA_MOD
#define BCF_FMA_MOD 3
#endif
#ifndef BCF_LANE_FMA_MOD
#define BCF_LANE_FMA_MOD 2
#endif
__host__ __device__ constexpr bool fma_pick(int i) { return BCF_FMA_MOD > 0 && (i % (BCF_FMA_MOD > 0 ? BCF_FMA_MOD : 1)) != 0; }
__host__ __device__ constexpr bool lane_fma_pick(int i) {
  return BCF_LANE_FMA_MOD > 0 && (i % (BCF_LANE_FMA_MOD > 0 ? BCF_LANE_FMA_MOD : 1)) != 0;
}

__device__ __forceinline__ void ce_keys(uint32_t& x, uint32_t& y, bool fma_max) {
  const uint32_t a = x, b = y;
  const uint32_t m = min(a, b);
  y = fma_max ? imad_u32(m, 0u - c_one, imad_u32(a, c_one, b)) : max(a, b);
  x = m;
}

template <bool PAIRS>
struct Elem;

template <>
struct Elem<false> {
  __device__ __forceinline__ static void ce(uint32_t& k0, uint32_t& k1, uint32_t&, uint32_t&,
                                            uint32_t&, uint32_t&) {
    const uint32_t lo = min(k0, k1);
    const uint32_t hi = max(k0, k1);
    k0 = lo;
    k1 = hi;
  }
};

template <>
struct Elem<true> {
  __device__ __forceinline__ static void ce(uint32_t& k0, uint32_t& k1, uint32_t& t0, uint32_t& t1,
                                            uint32_t& v0, uint32_t& v1) {
    const bool sw = (k1 < k0) || (k1 == k0 && t1 < t0);
    const uint32_t nk0 = sw ? k1 : k0, nk1 = sw ? k0 : k1;
    const uint32_t nt0 = sw ? t1 : t0, nt1 = sw ? t0 : t1;
    const uint32_t nv0 = sw ? v1 : v0, nv1 = sw ? v0 : v1;
    k0 = nk0; k1 = nk1; t0 = nt0; t1 = nt1; v0 = nv0; v1 = nv1;
  }
};

// Virtual-pad bookkeeping for networks padded from E to N = 2^ceil(log2 E):
// positions [E, N) hold virtual keys (-inf for the merger, +inf for the sort)
// whose comparisons resolve at compile time into moves.
template <int N>
struct PadMask {
  __host__ __device__ static constexpr unsigned all() { return N >= 32 ? 0xffffffffu : ((1u << N) - 1u); }
};

// Bitonic merger (Batcher) ascending over N = 2^ceil(log2 E) slots; slots
// [E, N) are virtual -inf.  Input must be bitonic (up-then-down, cyclically).
template <int E, bool PAIRS>
__device__ __forceinline__ void bitonic_merge_pad(uint32_t (&k)[E], uint32_t (&t)[E], uint32_t (&v)[E]) {
  constexpr int N = cpow2ceil(E);
  constexpr int LOGN = clog2(N);
  uint32_t K[N], Tg[N], V[N];
#pragma unroll
  for (int i = 0; i < N; ++i) {
    K[i] = i < E ? k[i] : 0u;
    if constexpr (PAIRS) { Tg[i] = i < E ? t[i] : 0u; V[i] = i < E ? v[i] : 0u; }
  }
  unsigned virt = PadMask<N>::all() & ~((E >= 32) ? 0xffffffffu : ((1u << E) - 1u));
#pragma unroll
  for (int ls = LOGN - 1; ls >= 0; --ls) {
    const int s = 1 << ls;
    unsigned nvirt = virt;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      if ((i & s) == 0) {
        const int j = i + s;
        const bool vi = (virt >> i) & 1u, vj = (virt >> j) & 1u;
        if (!vi && !vj) {
          if constexpr (PAIRS) Elem<PAIRS>::ce(K[i], K[j], Tg[i], Tg[j], V[i], V[j]);
          else ce_keys(K[i], K[j], fma_pick(i));  // compile-time after unrolling
        } else if (!vi && vj) {
          // min(-inf, x) = -inf goes to i, x moves to j
          K[j] = K[i];
          if constexpr (PAIRS) { Tg[j] = Tg[i]; V[j] = V[i]; }
          nvirt = (nvirt | (1u << i)) & ~(1u << j);
        }
      }
    }
    virt = nvirt;
  }
  // the N-E virtual -inf ended at slots [0, N-E): real outputs are [N-E, N)
#pragma unroll
  for (int i = 0; i < E; ++i) {
    k[i] = K[N - E + i];
    if constexpr (PAIRS) { t[i] = Tg[N - E + i]; v[i] = V[N - E + i]; }
  }
}

// Batcher odd-even merge sort ascending over N = 2^ceil(log2 E) slots; slots
// [E, N) are virtual +inf.  Used for the per-thread sort of E keys in the block
// sort (the paper uses Thrust's odd-even transposition sort; any
// network producing the same result is acceptable, reading c15).
template <int E, bool PAIRS>
__device__ __forceinline__ void oddeven_sort_pad(uint32_t (&k)[E], uint32_t (&t)[E], uint32_t (&v)[E]) {
  constexpr int N = cpow2ceil(E);
  constexpr int LOGN = clog2(N);
  uint32_t K[N], Tg[N], V[N];
#pragma unroll
  for (int i = 0; i < N; ++i) {
    K[i] = i < E ? k[i] : 0u;
    if constexpr (PAIRS) { Tg[i] = i < E ? t[i] : 0u; V[i] = i < E ? v[i] : 0u; }
  }
  unsigned virt = PadMask<N>::all() & ~((E >= 32) ? 0xffffffffu : ((1u << E) - 1u));
#pragma unroll
  for (int lp = 0; lp < LOGN; ++lp) {
    const int p = 1 << lp;
#pragma unroll
    for (int lk = lp; lk >= 0; --lk) {
      const int kk = 1 << lk;
      const int j0 = (kk == p) ? 0 : kk;  // kk % p
      unsigned nvirt = virt;
#pragma unroll
      for (int x = 0; x < N; ++x) {
        const int y = x + kk;
        if (x >= j0 && ((x - j0) % (2 * kk)) < kk && y < N && (x / (2 * p)) == (y / (2 * p))) {
          const bool vx = (virt >> x) & 1u, vy = (virt >> y) & 1u;
          if (!vx && !vy) {
            if constexpr (PAIRS) Elem<PAIRS>::ce(K[x], K[y], Tg[x], Tg[y], V[x], V[y]);
            else ce_keys(K[x], K[y], fma_pick(x));
          } else if (vx && !vy) {
            // max(+inf, y) = +inf goes to y, y's value moves to x
            K[x] = K[y];
            if constexpr (PAIRS) { Tg[x] = Tg[y]; V[x] = V[y]; }
            nvirt = (nvirt | (1u << y)) & ~(1u << x);
          }
        }
      }
      virt = nvirt;
    }
  }
#pragma unroll
  for (int i = 0; i < E; ++i) {
    k[i] = K[i];
    if constexpr (PAIRS) { t[i] = Tg[i]; v[i] = V[i]; }
  }
}

// ---------------------------------------------------------------------------
// In-register merge of the gathered registers (PAPER.md:354 uses Thrust's
// odd-even transposition sort; reading c15 allows any data-oblivious network
// with the same result).  items[] holds, circularly from k = a mod E,
// A_i ascending then B_i descending (bitonic).
//   E = 2^x: the bitonic merger sorts any cyclic shift directly.
//   otherwise: barrel-rotate left by k (static stages), pad with -inf, merge.
// Pairs: tag = rank in the stable order of A_i ++ B_i (pads: E).
// ---------------------------------------------------------------------------
template <int E, bool PAIRS>
__device__ __forceinline__ void merge_registers(uint32_t (&key)[E], uint32_t (&val)[E], int a, int nA,
                                                int nB) {
  const int k = a % E;
  uint32_t tag[E];
  if constexpr (is_pow2(E)) {
    if constexpr (PAIRS) {
#pragma unroll
      for (int j = 0; j < E; ++j) {
        int ia = j - k;
        if (ia < 0) ia += E;
        const int ib = E - 1 - ia;
        tag[j] = ia < nA ? (uint32_t)ia : (ib < nB ? (uint32_t)(nA + ib) : (uint32_t)E);
      }
    }
    bitonic_merge_pad<E, PAIRS>(key, tag, val);
  } else if constexpr (cpow2ceil(E) == E + 1 && !PAIRS) {
    // keys only, N = E + 1: append a copy X of register E-1 at slot E.  In the
    // circular order slot E sits between registers E-1 and 0, and X equals
    // one of its neighbours, so the 16 slots stay (circularly) bitonic.  After
    // the merger, drop one copy of X: out[i] = s[i] if s[i] < X else s[i+1].
    constexpr int N = E + 1;
    uint32_t K[N], Tg[N], V[N];
#pragma unroll
    for (int m = 0; m < E; ++m) K[m] = key[m];
    K[E] = key[E - 1];
    const uint32_t X = key[E - 1];
    bitonic_merge_pad<N, false>(K, Tg, V);
#pragma unroll
    for (int i = 0; i < E; ++i) key[i] = K[i] < X ? K[i] : K[i + 1];
  } else if constexpr (cpow2ceil(E) == E + 1) {
    // N = E + 1: insert one minimum element (key 0, tag 0; real tags shift
    // by 1) at register k, i.e. between the circular minimum candidates
    // B_i[0] (register k-1) and A_i[0] (register k).  The 16-register
    // circular sequence stays bitonic, and its sorted slot 0 is the insert,
    // dropped afterwards.  Costs 2 selects per register instead of a
    // log2(E)-stage barrel rotation.
    constexpr int N = E + 1;
    uint32_t K[N], Tg[N], V[N];
#pragma unroll
    for (int m = 0; m < N; ++m) {
      const uint32_t lo = m < E ? key[m] : 0u;
      const uint32_t hi = m >= 1 ? key[m - 1] : 0u;
      K[m] = m < k ? lo : (m == k ? 0u : hi);
      if constexpr (PAIRS) {
        const uint32_t vlo = m < E ? val[m] : 0u;
        const uint32_t vhi = m >= 1 ? val[m - 1] : 0u;
        V[m] = m < k ? vlo : (m == k ? 0u : vhi);
        // tag of the element now in slot m (its register before insertion)
        const int j = m < k ? m : m - 1;
        int ia = j - k;
        if (ia < 0) ia += E;
        const int ib = E - 1 - ia;
        const uint32_t t = ia < nA ? (uint32_t)ia + 1u : (ib < nB ? (uint32_t)(nA + ib) + 1u : (uint32_t)E + 1u);
        Tg[m] = m == k ? 0u : t;
      }
    }
    bitonic_merge_pad<N, PAIRS>(K, Tg, V);
#pragma unroll
    for (int i = 0; i < E; ++i) {
      key[i] = K[i + 1];
      if constexpr (PAIRS) val[i] = V[i + 1];
    }
  } else {
    // rotate left by k: new[m] = old[(m + k) mod E] (barrel, static selects)
    constexpr int NBITS = clog2(E - 1) + 1;  // bits of k in [0, E-1]
#pragma unroll
    for (int bit = 0; bit < NBITS; ++bit) {
      const int sh = 1 << bit;
      const bool b = (k >> bit) & 1;
      uint32_t tk[E], tv[E];
#pragma unroll
      for (int m = 0; m < E; ++m) {
        tk[m] = b ? key[(m + sh) % E] : key[m];
        if constexpr (PAIRS) tv[m] = b ? val[(m + sh) % E] : val[m];
      }
#pragma unroll
      for (int m = 0; m < E; ++m) {
        key[m] = tk[m];
        if constexpr (PAIRS) val[m] = tv[m];
      }
    }
    if constexpr (PAIRS) {
#pragma unroll
      for (int m = 0; m < E; ++m) {
        const int ib = E - 1 - m;
        tag[m] = m < nA ? (uint32_t)m : (ib < nB ? (uint32_t)(nA + ib) : (uint32_t)E);
      }
    }
    bitonic_merge_pad<E, PAIRS>(key, tag, val);
  }
}

// ---------------------------------------------------------------------------
// Warp phase of the block sort (keys only, E + 1 = w = 32): the first five
// merge levels (runs of 1, 2, 4, 8, 16 threads -> runs of one warp) merge
// registers across lanes with shuffles instead of going through shared
// memory, so they cannot have bank conflicts at all and cost (L+1) shuffle
// stages + one in-register bitonic merger at level L instead of a shared
// scatter / split search / gather.  Every lane holds 32 slots: its E sorted
// keys and one pad (max key) in slot E.  A level merges the ascending runs of
// lanes [b, b+h) and [b+h, b+2h) (h = 2^L): a flip stage (slot i of lane t
// against slot 31-i of lane t ^ (2h-1): the two ascending runs read as one
// bitonic sequence), half-cleaners across lanes (distance h/2 .. 1), then the
// 32-slot bitonic merger inside each lane.  Keys only: equal keys are equal
// bits, so the (unstable) network's order among them is unobservable.
// After level 4 the warp's 1024 slots are ascending: lanes 0..30 hold its
// 992 keys (32 each), lane 31 holds the 32 pads.
// ---------------------------------------------------------------------------
// lane keeps min(a, p) (hi = 0) or max(a, p) (hi = 1).  fma form: one ALU
// min + three FMA-pipe IMADs, r = m + hi * (a + p - 2m); else two ALU ops.
__device__ __forceinline__ uint32_t lane_minmax(uint32_t a, uint32_t p, bool hi, uint32_t hi01, bool fma_form) {
  if (fma_form) {
    const uint32_t m = min(a, p);
    return imad_u32(hi01, imad_u32(m, 0u - 2u * c_one, imad_u32(a, c_one, p)), m);
  }
  return hi ? max(a, p) : min(a, p);
}

template <int NS = W>
__device__ __forceinline__ void warp_bitonic_levels(uint32_t (&k)[NS], int lane) {
#pragma unroll
  for (int L = 0; L < 5; ++L) {
    const bool up = (lane >> L) & 1;
    const uint32_t up01 = up ? 1u : 0u;
    const int m = (2 << L) - 1;
#pragma unroll
    for (int i = 0; i < NS / 2; ++i) {
      const int j = NS - 1 - i;
      const uint32_t pi = __shfl_xor_sync(FULL, k[j], m);
      const uint32_t pj = __shfl_xor_sync(FULL, k[i], m);
      k[i] = lane_minmax(k[i], pi, up, up01, false);
      k[j] = lane_minmax(k[j], pj, up, up01, true);
    }
#pragma unroll
    for (int d = L - 1; d >= 0; --d) {
      const bool hi = (lane >> d) & 1;
      const uint32_t hi01 = hi ? 1u : 0u;
#pragma unroll
      for (int i = 0; i < NS; ++i) {
        const uint32_t p = __shfl_xor_sync(FULL, k[i], 1 << d);
        k[i] = lane_minmax(k[i], p, hi, hi01, lane_fma_pick(i));
      }
    }
    uint32_t dt[NS], dv[NS];
    bitonic_merge_pad<NS, false>(k, dt, dv);
  }
}

// Conflict-free write of a warp's sorted 992-key run (lanes 0..30 x 32 slots)
// into the block sort's level-5 layout: the A run (even warp of a merge
// group) ascending at [gbase, gbase + S), the B run reversed (pi) ending at
// gbase + 2S (S = 32E).  16-byte stores: in round r lane t writes its quad
// (r + t) mod 8, so the 8 lanes of each quarter-warp phase hit 8 distinct
// 16-byte bank groups (the quads are brought into round order by a 3-stage
// barrel rotation of the registers).
template <int E>
__device__ __forceinline__ void warp_run_scatter(uint32_t* __restrict__ sk, const uint32_t (&k)[W], int warp,
                                                 int lane) {
  static_assert(E + 1 == W, "warp phase needs E = 31");
  constexpr int S = W * E;
  uint32_t r[W];
#pragma unroll
  for (int i = 0; i < W; ++i) r[i] = k[i];
#pragma unroll
  for (int b = 0; b < 3; ++b) {
    const bool on = (lane >> b) & 1;
    uint32_t t[W];
#pragma unroll
    for (int i = 0; i < W; ++i) t[i] = on ? r[(i + (4 << b)) % W] : r[i];
#pragma unroll
    for (int i = 0; i < W; ++i) r[i] = t[i];
  }
  if (lane == W - 1) return;  // the pads
  const int gbase = (warp >> 1) * 2 * S;
  const bool isB = warp & 1;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const int qq = (q + lane) & 7;
    if (isB) {
      uint4 v = make_uint4(r[4 * q + 3], r[4 * q + 2], r[4 * q + 1], r[4 * q]);
      *reinterpret_cast<uint4*>(sk + gbase + 2 * S - 4 - W * lane - 4 * qq) = v;
    } else {
      uint4 v = make_uint4(r[4 * q], r[4 * q + 1], r[4 * q + 2], r[4 * q + 3]);
      *reinterpret_cast<uint4*>(sk + gbase + W * lane + 4 * qq) = v;
    }
  }
}

// The same write for E = 16 or 8 (E slots per lane, no pads, rho != identity):
// lane i of warp run holds run positions [E i, E i + E); round r writes
// position E i + r (A, ascending) or its mirror 2S-1-(E i + r) (B, pi), a
// round set of the run's wE window (Lemma 1 / Cor. 3): conflict-free via rho.
template <int E>
__device__ __forceinline__ void warp_run_scatter_rho(uint32_t* __restrict__ sk, const uint32_t (&k)[E], int warp,
                                                     int lane) {
  constexpr int S = W * E;
  const int gbase = (warp >> 1) * 2 * S;
  const bool isB = warp & 1;
  const int base = isB ? gbase + 2 * S - 1 - E * lane : gbase + E * lane;
  const int step = isB ? -1 : 1;
#pragma unroll
  for (int r = 0; r < E; ++r) sk[rho<E>(base + step * r)] = k[r];
}

// The same for E < 16 other than 8 (16 slots per lane, 16 - E max-key pads; the
// warp's 32E real keys fill lanes 0..2E-1): lane i's slots are rotated by
// sigma_i, so that in round s it writes run position 16 i + (s + sigma_i) mod 16.
// Through rho, bank(k) = (k + (k / P mod d)) mod 32 (P = wE/d = 0 mod 32): a
// search over sigma (2E lanes x 16 rounds, A and mirrored B positions) found
// sigma_i = i / 2 conflict-free for E = 10 and 12, and the same with
// sigma_3 = 7 for E = 14; for odd E (rho = identity) sigma_i = i / 2 gives the
// banks 16 (i mod 2) + (s + i / 2) mod 16, distinct for 2E <= 30 lanes.
template <int E>
__device__ __forceinline__ void warp_run_scatter_rho_pad(uint32_t* __restrict__ sk, const uint32_t (&k)[16], int warp,
                                                         int lane) {
  static_assert(E <= 15 && E != 8, "padded warp phase: E < 16 (E = 8 has no pads)");
  constexpr int S = W * E;
  const int sigma = (E == 14 && lane == 3) ? 7 : (lane >> 1);
  uint32_t r[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) r[i] = k[i];
#pragma unroll
  for (int b = 0; b < 4; ++b) {
    const bool on = (sigma >> b) & 1;
    uint32_t t[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) t[i] = on ? r[(i + (1 << b)) & 15] : r[i];
#pragma unroll
    for (int i = 0; i < 16; ++i) r[i] = t[i];
  }
  // r[s] holds slot (s + sigma) mod 16
  if (lane >= 2 * E) return;  // only pads
  const int gbase = (warp >> 1) * 2 * S;
  const bool isB = warp & 1;
#pragma unroll
  for (int s = 0; s < 16; ++s) {
    const int pos = 16 * lane + ((s + sigma) & 15);
    sk[rho<E>(isB ? gbase + 2 * S - 1 - pos : gbase + pos)] = r[s];
  }
}

// f32 <-> order-preserving u32 (IEEE totalOrder, reading c2)
__device__ __forceinline__ uint32_t f32_encode(uint32_t b) {
  return b ^ ((uint32_t)((int32_t)b >> 31) | 0x80000000u);
}
__device__ __forceinline__ uint32_t f32_decode(uint32_t u) {
  return u ^ ((~(uint32_t)((int32_t)u >> 31)) | 0x80000000u);
}

}  // namespace bcf
