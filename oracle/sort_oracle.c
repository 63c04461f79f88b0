/*
 * oracle/sort_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously correct CPU reference for what the CUDA path computes:
 * a stable sort of n 4-byte keys (§1 "Thrust's mergesort
 * implementation", §5 "pairwise merge sort provided in Thrust",
 * PAPER.md:356 "4-byte integers").  A stable sort is unique given the order, so
 * the oracle is the plain definition written out as a textbook top-down
 * mergesort whose merge takes from the right run only when its head is strictly
 * smaller ("ties go to the left run").
 *
 * Key orders:
 *   u32   numeric order;
 *   f32   IEEE 754-2008 §5.10 totalOrder, written from its definition on the
 *         sign and the magnitude bits (NOT via the product's XOR encoding);
 *   pairs stable by u32 key, values carried along.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares no code with the
 * CUDA path (paper_conf_spaa_berneys25_b200/csrc).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- key comparisons: "a strictly before b" ---------------------------- */

static int less_u32(uint32_t a, uint32_t b) { return a < b; }

/* IEEE 754 totalOrder on binary32 bit patterns.
 * - a negative-signed datum orders below a positive-signed one (so -0 < +0,
 *   -NaN < everything, +NaN > everything);
 * - two positive-signed data order by their magnitude bits ascending
 *   (+0 < denormals < normals < +inf < +NaN payloads ascending);
 * - two negative-signed data order by their magnitude bits descending. */
static int less_f32_total(uint32_t a, uint32_t b) {
    uint32_t sa = a >> 31, sb = b >> 31;
    uint32_t ma = a & 0x7FFFFFFFu, mb = b & 0x7FFFFFFFu;
    if (sa != sb) return sa > sb;      /* negative before positive */
    if (sa == 0) return ma < mb;       /* both positive */
    return ma > mb;                    /* both negative */
}

typedef int (*less_fn)(uint32_t, uint32_t);

/* ---- top-down stable mergesort ------------------------------------------ */

static void merge_runs(uint32_t *k, uint32_t *v, uint32_t *tk, uint32_t *tv,
                       uint64_t lo, uint64_t mid, uint64_t hi, less_fn less) {
    uint64_t i = lo, j = mid, o = lo;
    while (i < mid && j < hi) {
        /* take from the right run only if strictly smaller: ties to the left */
        if (less(k[j], k[i])) {
            tk[o] = k[j];
            if (v) tv[o] = v[j];
            ++j;
        } else {
            tk[o] = k[i];
            if (v) tv[o] = v[i];
            ++i;
        }
        ++o;
    }
    while (i < mid) { tk[o] = k[i]; if (v) tv[o] = v[i]; ++i; ++o; }
    while (j < hi)  { tk[o] = k[j]; if (v) tv[o] = v[j]; ++j; ++o; }
    memcpy(k + lo, tk + lo, (size_t)(hi - lo) * sizeof(uint32_t));
    if (v) memcpy(v + lo, tv + lo, (size_t)(hi - lo) * sizeof(uint32_t));
}

static void msort(uint32_t *k, uint32_t *v, uint32_t *tk, uint32_t *tv,
                  uint64_t lo, uint64_t hi, less_fn less) {
    if (hi - lo < 2) return;
    uint64_t mid = lo + (hi - lo) / 2;
    msort(k, v, tk, tv, lo, mid, less);
    msort(k, v, tk, tv, mid, hi, less);
    merge_runs(k, v, tk, tv, lo, mid, hi, less);
}

static int sort_generic(const uint32_t *kin, const uint32_t *vin, uint32_t *kout,
                        uint32_t *vout, uint64_t n, less_fn less) {
    if (n == 0) return 0;
    if (kout != kin) memmove(kout, kin, (size_t)n * sizeof(uint32_t));
    if (vout && vin && vout != vin) memmove(vout, vin, (size_t)n * sizeof(uint32_t));
    uint32_t *tk = (uint32_t *)malloc((size_t)n * sizeof(uint32_t));
    uint32_t *tv = vout ? (uint32_t *)malloc((size_t)n * sizeof(uint32_t)) : NULL;
    if (!tk || (vout && !tv)) { free(tk); free(tv); return -1; }
    msort(kout, vout, tk, tv, 0, n, less);
    free(tk);
    free(tv);
    return 0;
}

/* ---- exported entry points (ctypes) ------------------------------------- */

int oracle_sort_u32(const uint32_t *in, uint32_t *out, uint64_t n) {
    return sort_generic(in, NULL, out, NULL, n, less_u32);
}

/* f32 keys are passed as their bit patterns */
int oracle_sort_f32(const uint32_t *in_bits, uint32_t *out_bits, uint64_t n) {
    return sort_generic(in_bits, NULL, out_bits, NULL, n, less_f32_total);
}

int oracle_sort_pairs_u32(const uint32_t *kin, const uint32_t *vin, uint32_t *kout,
                          uint32_t *vout, uint64_t n) {
    return sort_generic(kin, vin, kout, vout, n, less_u32);
}

/* 1 if a is strictly before b in IEEE totalOrder (exposed for the pins) */
int oracle_f32_total_less(uint32_t a, uint32_t b) { return less_f32_total(a, b); }
