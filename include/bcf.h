/*
 * bcf.h -- C ABI of the B200-native bank-conflict-free mergesort.
 *
 * Implements the hot path of K. Berney, N. Sitchinava, "Eliminating Bank
 * Conflicts in GPU Mergesort", SPAA '25 (cited as PAPER.md:<line>):
 * Thrust-style stable pairwise mergesort (PAPER.md:59-61 §1, :348-354 §5)
 * whose shared-memory tiles use the paper's permutation rho(A u pi(B))
 * (Alg. 1 line 2; §3.1-3.3) and the load-balanced dual
 * subsequence gather (Alg. 1), so that no input causes a
 * shared-memory bank conflict.
 *
 * Conventions (all entry points):
 *  - Pointers named d_* are DEVICE pointers (cudaMalloc / torch CUDA tensors)
 *    on the current device; h_* are HOST pointers.  The caller owns all
 *    memory; the library never allocates device memory.
 *  - Temporary storage is queried CUB-style: call with d_temp == NULL to get
 *    *temp_bytes, then call again with a buffer of at least that size.
 *  - All device work is enqueued on `stream` (may be 0 = legacy default
 *    stream) and is asynchronous; nothing synchronizes the host, except
 *    bcf_profile_collect.
 *  - Argument errors are returned synchronously before any launch.
 *    n > 0 with a NULL data pointer -> BCF_ERROR_INVALID_VALUE; a temp buffer
 *    smaller than required -> BCF_ERROR_TEMP_TOO_SMALL; (E, u) outside the
 *    instantiated set -> BCF_ERROR_UNSUPPORTED.  Launch / runtime errors
 *    return BCF_ERROR_CUDA and bcf_last_cuda_error() gives the cudaError_t
 *    (thread-local).  No C++ exception crosses this boundary.
 *  - n = 0 is a no-op; d_in == d_out (in place) is allowed.
 *  - n is 64-bit; sizes up to 2^32 keys are supported (bounded by memory).
 *  - Thread-safe: no mutable global state except the optional profiler.
 */
#ifndef BCF_H_
#define BCF_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BCF_ABI_VERSION 1

typedef enum {
  BCF_SUCCESS = 0,
  BCF_ERROR_INVALID_VALUE = 1,
  BCF_ERROR_UNSUPPORTED = 2,
  BCF_ERROR_CUDA = 3,
  BCF_ERROR_TEMP_TOO_SMALL = 4
} bcf_status;

typedef enum {
  /* the paper's bank-conflict-free design (CF-Merge) */
  BCF_ALGO_CONFLICT_FREE = 0,
  /* the unmodified Thrust design the paper compares against (A|B forward in
     shared memory, per-thread merge-path binary search, serial merge reading
     shared memory).  Keys only (u32 / f32). */
  BCF_ALGO_BASELINE = 1
} bcf_algo;

/* "software parameters" E and u: items per thread and threads
   per block.  0 selects the default.  Instantiated set: E in [7, 17] or
   E = 31, u in {128, 256, 512}. */
typedef struct {
  int32_t items_per_thread; /* E */
  int32_t block_threads;    /* u */
  int32_t algo;             /* bcf_algo */
} bcf_params;

/* Default (E, u) chosen for sm_100a by measurement: keys
   (u32 / f32) (31, 128); pairs (11, 256).  A zero field in the params passed
   to a sort selects that entry point's default. */
void bcf_default_params(bcf_params* p);
void bcf_default_pairs_params(bcf_params* p);

/* Stable sort of n u32 keys, ascending ("4-byte
   integers").  d_in is not modified unless d_in == d_out.
   Temp: n keys (+ alignment).  p may be NULL (defaults). */
bcf_status bcf_sort_u32(const uint32_t* d_in, uint32_t* d_out, uint64_t n, void* d_temp,
                        size_t* temp_bytes, const bcf_params* p, void* stream);

/* Sort n f32 keys by IEEE 754 totalOrder (-NaN < -inf < ... < -0 < +0 < ...
   < +inf < +NaN; reading c2).  Keys are encoded to order-preserving
   u32 on the first load and decoded on the final store (fused, no extra
   pass).  Ties are bit-identical, so stability is unobservable. */
bcf_status bcf_sort_f32(const float* d_in, float* d_out, uint64_t n, void* d_temp,
                        size_t* temp_bytes, const bcf_params* p, void* stream);

/* The pass plan a sort of n keys (pairs != 0: pairs) with params p runs
   (host only, no CUDA call): block-sort tile (keys per block-sort CTA; the
   keys-only CF default (31, 128) sorts tiles of 2u threads), merge-pass tile
   u*E, and the number of pairwise merge passes ceil(log2(n / block tile)). */
bcf_status bcf_sort_plan(uint64_t n, const bcf_params* p, int32_t pairs, int64_t* block_sort_tile,
                         int64_t* merge_tile, int32_t* merge_passes);

/* End-to-end sort of nbatch independent HOST arrays of n u32 keys each:
   h_in[i] -> (H2D) -> bcf_sort_u32 -> (D2H) -> h_out[i] (h_out[i] may equal
   h_in[i]; the h_in/h_out pointer arrays are host arrays).  Two device slots:
   the H2D copy of batch i+1 and the D2H copy of batch i-1 run on the
   library's own copy streams while batch i sorts on `stream`, so the
   throughput is bounded by max(H2D, sort, D2H) per batch.  Host buffers
   should be pinned (cudaHostAlloc / torch pin_memory) for the copies to be
   asynchronous; pageable memory is correct but serialises.  Temp (CUB-style
   query with d_temp = NULL): 4 n keys + the sort's temp.  Stream-ordered:
   the work starts after the work already queued on `stream`, and `stream`
   completes after the last read-back (synchronise it before reading h_out). */
bcf_status bcf_sort_u32_host_batch(const uint32_t* const* h_in, uint32_t* const* h_out, int32_t nbatch,
                                   uint64_t n, void* d_temp, size_t* temp_bytes, const bcf_params* p,
                                   void* stream);

/* Stable sort of (key, value) pairs by u32 key; values (u32) follow their
   keys; equal keys keep their input order.  Temp: n keys + n values.
   BCF_ALGO_BASELINE is not supported for pairs (BCF_ERROR_UNSUPPORTED). */
bcf_status bcf_sort_pairs_u32(const uint32_t* d_keys_in, uint32_t* d_keys_out,
                              const uint32_t* d_vals_in, uint32_t* d_vals_out, uint64_t n,
                              void* d_temp, size_t* temp_bytes, const bcf_params* p, void* stream);

/* Worst-case input for the unmodified Thrust mergesort with parameters
   (E, u) (Section 4: sequences S and T, Theorem 8; inside a
   mixed thread the x part is read first and the y part last, DESIGN.md
   reading c9; multi-level composition per reading c10).  Writes a
   permutation of 0..n-1 to d_out.  Deterministic in (n, E, u, seed).
   Generated on the device as a closed form of the position (one thread per
   run of E keys walks the merge levels up), stream-ordered, no host sync, no
   host memory: any n up to 2^36.  E in [2, 32], u a power of two >= 32;
   otherwise BCF_ERROR_UNSUPPORTED. */
bcf_status bcf_worst_case_u32(uint32_t* d_out, uint64_t n, int32_t E, int32_t u, uint64_t seed,
                              void* stream);
/* Same construction into host memory (no CUDA call). */
bcf_status bcf_worst_case_u32_host(uint32_t* h_out, uint64_t n, int32_t E, int32_t u,
                                   uint64_t seed);

/* Distributed-sort phases (the exchange itself is done by torch.distributed).
   For each of npiv pivots v (device array), count the keys of the sorted
   run d_sorted[0, n) that are < v and <= v (binary searches, one thread per
   pivot).  Outputs are device arrays of npiv u64. */
bcf_status bcf_split_counts_u32(const uint32_t* d_sorted, uint64_t n, const uint32_t* d_pivots,
                                int32_t npiv, uint64_t* d_lt_counts, uint64_t* d_le_counts,
                                void* stream);

/* Stable merge of nruns ascending sorted runs stored back to back in d_runs
   (run r = [h_run_offsets[r], h_run_offsets[r+1]), host array of nruns+1
   entries, h_run_offsets[0] = 0); equal keys keep run order (run 0 first).
   Output ascending in d_out (must not alias d_runs).  Pairwise passes of the
   same CF merge kernel.  Values: pass NULL for keys only. */
bcf_status bcf_merge_runs_u32(const uint32_t* d_runs, const uint32_t* d_run_vals,
                              const uint64_t* h_run_offsets, int32_t nruns, uint32_t* d_out,
                              uint32_t* d_out_vals, void* d_temp, size_t* temp_bytes,
                              const bcf_params* p, void* stream);

/* bcf_merge_runs_u32 for runs anywhere in device memory, keys only: run r is
   h_run_ptrs[r][0, h_run_lens[r]) (host arrays of nruns entries; the
   pointers may be peer-mapped memory of other GPUs, bcf_ipc_open).  The
   first pairwise pass reads every run through its own pointer (over NVLink
   for a peer's run), so an all-to-all exchange followed by the run merge
   becomes one pass that moves each key once; later
   passes are local.  Equal keys keep run order (run 0 first).  nruns <= 4096.
   Temp: CUB-style query, as bcf_merge_runs_u32 of the same lengths.  The
   caller orders the producers of peer runs before this call (e.g. stream
   synchronise + barrier) and keeps them alive until it completes. */
bcf_status bcf_merge_runs_ptrs_u32(const uint32_t* const* h_run_ptrs, const uint64_t* h_run_lens,
                                   int32_t nruns, uint32_t* d_out, void* d_temp, size_t* temp_bytes,
                                   const bcf_params* p, void* stream);

/* CUDA IPC for bcf_merge_runs_ptrs_u32 across the processes of one node
   (one process per GPU).  bcf_ipc_export: the handle (BCF_IPC_HANDLE_BYTES
   bytes written to `handle`) of the allocation holding d_ptr and d_ptr's
   byte offset in it.  bcf_ipc_open: map a peer's handle (peer access enabled
   lazily); *d_base = the allocation's base in this process.  bcf_ipc_close:
   unmap. */
#define BCF_IPC_HANDLE_BYTES 64
bcf_status bcf_ipc_export(const void* d_ptr, void* handle, uint64_t* offset);
bcf_status bcf_ipc_open(const void* handle, void** d_base);
bcf_status bcf_ipc_close(void* d_base);

/* Stable merge of two ascending sorted arrays A = d_a[0, na) and
   B = d_b[0, nb) into d_out[0, na+nb) (must alias neither); equal keys: all
   of A's before B's.  The merge step of the pairwise mergesort (merge path,
   PAPER.md:59-61) as a primitive -- "any parallel scan of a pair of arrays"
    -- run as ONE pass of the CF merge kernel (conflict-free
   staging rho(A u pi(B)) and Alg. 1 gather), so no input
   pair causes a bank conflict.  Values: pass d_a_vals = d_b_vals =
   d_out_vals = NULL for keys only, else all three (values follow keys).
   Precondition: A and B ascending (not checked -- that would cost a pass;
   unsorted inputs are undefined behaviour, as for any merge-path merge).
   Paths: E coprime with 32, d_a 16-byte aligned (pairs: also d_a_vals
   16-byte aligned and d_out / d_out_vals at the same 16-byte phase): B (and
   its values) is first reversed into temp (the persistent window kernel
   bulk-copies B windows into their reversed slots, so it needs B stored
   descending: +8 B of traffic per B key, +8 B per B value), then one pass of
   the window kernel; otherwise one pass of the plain LSU-staged CF kernel
   reading B ascending.  Temp (CUB-style query): 512 bytes (group
   descriptor) + 4 (nb + 8) bytes rounded up to 256, twice that for pairs.
   na = nb = 0 is a no-op; one side empty is a device copy.  Only
   BCF_ALGO_CONFLICT_FREE.  Kernel launches only (the group descriptor is
   written by a 1-thread kernel), so the call can be captured into a CUDA
   graph, like the sorts -- after one earlier uncaptured call with the same
   (E, u) on the device: the first launch of each kernel sets its shared
   memory attribute and queries its occupancy, which capture does not allow.
   bcf_merge_runs_u32 writes its per-pass descriptor tables with small
   kernels too and is capturable under the same condition. */
bcf_status bcf_merge_u32(const uint32_t* d_a, uint64_t na, const uint32_t* d_b, uint64_t nb,
                         const uint32_t* d_a_vals, const uint32_t* d_b_vals, uint32_t* d_out,
                         uint32_t* d_out_vals, void* d_temp, size_t* temp_bytes, const bcf_params* p,
                         void* stream);

/* Set operations of two ascending u32 sequences A = d_a[0, na) and
   B = d_b[0, nb) with the multiset semantics of ISO C++ [alg.set.operations]:
   for a key with m copies in A and n in B, union keeps all m copies from A
   and then the last max(n - m, 0) of B's, intersection the first min(m, n)
   of A's, difference (A - B) the last max(m - n, 0) of A's, symmetric
   difference the last m - n of A's or the last n - m of B's.  The output is
   ascending (equal keys: A's copies first).  The paper's generalisation of
   its technique to "any algorithm that involves a parallel scan of a pair of
   arrays": the pair is merged by the conflict-free merge
   (bcf_merge_u32 with source tags, ties to A), then the kept elements of
   every equal-key run are flagged and compacted in merged order.
   d_out (na + nb words) receives the kept keys, d_out_src (optional, NULL
   to skip) where each came from: the A index, or 0x80000000 | the B index;
   *d_count (DEVICE u64) their number.  na, nb < 2^31.  Precondition: A and B
   ascending (not checked).  Temp: CUB-style query. */
typedef enum {
  BCF_SET_UNION = 0,
  BCF_SET_INTERSECTION = 1,
  BCF_SET_DIFFERENCE = 2,
  BCF_SET_SYMMETRIC_DIFFERENCE = 3
} bcf_set_op;
bcf_status bcf_set_op_u32(int32_t op, const uint32_t* d_a, uint64_t na, const uint32_t* d_b, uint64_t nb,
                          uint32_t* d_out, uint32_t* d_out_src, uint64_t* d_count, void* d_temp,
                          size_t* temp_bytes, const bcf_params* p, void* stream);

const char* bcf_status_string(bcf_status s);
int32_t bcf_abi_version(void);
/* cudaError_t (as int) of the last BCF_ERROR_CUDA on the calling thread */
int32_t bcf_last_cuda_error(void);

/* ---- measurement hooks (bench.py) ----------------------------------------
   When enabled, every kernel launched by the library is bracketed by CUDA
   events recorded on the launch stream; bcf_profile_collect synchronizes
   those events and returns, per kernel class, the number of launches and the
   summed device milliseconds.  Disabled by default (zero overhead). */
typedef struct {
  char name[32];     /* "block_sort", "merge_pass", "split_counts", ... */
  int64_t launches;
  double total_ms;
  uint64_t keys;     /* keys processed by those launches (sum of n) */
} bcf_kernel_stats;

bcf_status bcf_profile_enable(int32_t on);
/* fills up to max entries, *count = number of classes; resets the record */
bcf_status bcf_profile_collect(bcf_kernel_stats* out, int32_t max, int32_t* count);
/* total kernels launched by this process through the library (always on) */
int64_t bcf_launch_count(void);
/* debug: copy the per-CTA timeline recorded for merge pass $BCF_TRACE (globaltimer
   ns; 256 slots per CTA) into host memory; BCF_ERROR_INVALID_VALUE if none */
bcf_status bcf_debug_trace_copy(void* host, uint64_t bytes);

#ifdef __cplusplus
}
#endif

#endif /* BCF_H_ */
