/*
 * oracle/setops_oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
 *
 * Set operations on two ascending u32 sequences with multiset semantics: the
 * "parallel scan of a pair of arrays" the paper generalises its technique to
 * (§6: "our approach can be used to convert any algorithm that
 * involves a parallel scan of a pair of arrays into a bank conflict free
 * algorithm").  The paper gives no definition of the operations, so the oracle
 * is the C++ standard's (ISO C++ [alg.set.operations]) written out as a plain
 * two-pointer walk over the equal-key runs:
 *   for a key with m copies in A and n copies in B,
 *   union                 all m copies from A, then the LAST max(n - m, 0) of B's;
 *   intersection          the FIRST min(m, n) copies from A;
 *   difference (A - B)    the LAST max(m - n, 0) copies from A;
 *   symmetric difference  the last m - n from A if m > n, the last n - m from B if n > m.
 * Output ascending; out_src (optional) records where each output came from:
 * the A index, or 0x80000000 | the B index.
 * Shares no code with the CUDA path.
 */
#include <stdint.h>

enum { OP_UNION = 0, OP_INTERSECTION = 1, OP_DIFFERENCE = 2, OP_SYMMETRIC_DIFFERENCE = 3 };

static void emit(uint32_t *out, uint32_t *src, uint64_t *o, uint32_t key, uint32_t tag) {
    out[*o] = key;
    if (src) src[*o] = tag;
    ++*o;
}

int oracle_set_op_u32(int op, const uint32_t *a, uint64_t na, const uint32_t *b, uint64_t nb,
                      uint32_t *out, uint32_t *out_src, uint64_t *count) {
    uint64_t i = 0, j = 0, o = 0, k;
    if (op < 0 || op > 3) return -1;
    while (i < na || j < nb) {
        if (j == nb || (i < na && a[i] < b[j])) {          /* key only in A (here) */
            if (op != OP_INTERSECTION) emit(out, out_src, &o, a[i], (uint32_t)i);
            ++i;
        } else if (i == na || b[j] < a[i]) {                /* key only in B */
            if (op == OP_UNION || op == OP_SYMMETRIC_DIFFERENCE)
                emit(out, out_src, &o, b[j], 0x80000000u | (uint32_t)j);
            ++j;
        } else {                                            /* equal keys: runs of m and n */
            const uint32_t x = a[i];
            uint64_t m = 0, n = 0;
            while (i + m < na && a[i + m] == x) ++m;
            while (j + n < nb && b[j + n] == x) ++n;
            switch (op) {
            case OP_UNION:
                for (k = 0; k < m; ++k) emit(out, out_src, &o, x, (uint32_t)(i + k));
                for (k = (n > m ? n - (n - m) : n); k < n; ++k)   /* last n - m of B's */
                    emit(out, out_src, &o, x, 0x80000000u | (uint32_t)(j + k));
                break;
            case OP_INTERSECTION:
                for (k = 0; k < (m < n ? m : n); ++k) emit(out, out_src, &o, x, (uint32_t)(i + k));
                break;
            case OP_DIFFERENCE:
                for (k = (m > n ? n : m); k < m; ++k) emit(out, out_src, &o, x, (uint32_t)(i + k));
                break;
            default:
                if (m > n)
                    for (k = n; k < m; ++k) emit(out, out_src, &o, x, (uint32_t)(i + k));
                else
                    for (k = m; k < n; ++k) emit(out, out_src, &o, x, 0x80000000u | (uint32_t)(j + k));
            }
            i += m;
            j += n;
        }
    }
    *count = o;
    return 0;
}
