/*
 * ptas_oracle_omp.c — the paper's CPU comparator shape (Alg 2, the OpenMP DP
 * of Ghalami & Grosu [1]) for the cpu_baseline leg of
 * bench.py, run on all host cores.
 *
 * TEST INFRASTRUCTURE ONLY (like ptas_oracle.c): only tests/ and bench.py's
 * cpu_baseline leg may load it.  It shares no code with the product library
 * and none with ptas_oracle.c either (it is checked against oracle_dp entry
 * by entry in tests/test_oracle_pins.py, and oracle_dp is pinned by brute
 * force, exhaustive bin packing and closed forms).
 *
 * Alg 2, step by step:
 *   l.2      sigma = prod (N_i + 1)
 *   l.3      entries in row-major order, last class fastest
 *   l.4–8    d_i = sum of the digits of entry i (its level)
 *   l.10–25  for l = 1 .. n': in parallel over the entries with d_i = l:
 *            generate the configurations s <= v with sum s_i r_i <= T,
 *            OPT(v) = 1 + min OPT(v - s)                 (Eq. 1)
 * Two departures from the literal Alg 2, neither changing any value:
 *   - the entries with d_i = l are gathered once by a counting sort on d
 *     (Alg 2 rescans all sigma entries at every level);
 *   - OPT(v - s) is read at row-major index idx(v) - off(s) instead of the
 *     table-wide search of l.18 (row-major indices are a plain definition).
 * The configuration set C(T) is enumerated once (Alg 2 l.17 regenerates it per
 * state; the set {s in C : s <= v} is the same).
 */
#include <stdint.h>
#include <stdlib.h>
#include <omp.h>

#define OMP_OK 0
#define OMP_EINVAL -1
#define OMP_ETOOBIG -2
#define OMP_ENOMEM -3

int oracle_omp_threads(void) { return omp_get_max_threads(); }

/* table[] (int32, sigma entries, row-major) receives OPT for every entry;
 * *relax_out counts the (v, s) pairs with s in C, s <= v. */
int oracle_dp_omp(const int32_t *N, const int64_t *r, int32_t K, int64_t T,
                  int32_t *table, int64_t table_cap, int32_t *optN, double *relax_out)
{
    if (K < 0 || K > 64) return OMP_EINVAL;
    int64_t sigma = 1;
    int32_t levels = 0;
    for (int32_t i = 0; i < K; i++) {
        if (N[i] < 0 || r[i] < 1 || (N[i] > 0 && r[i] > T)) return OMP_EINVAL;
        if (sigma > INT64_MAX / (N[i] + 1)) return OMP_ETOOBIG;
        sigma *= (N[i] + 1);
        levels += N[i];
    }
    if (sigma > table_cap) return OMP_ETOOBIG;
    table[0] = 0;
    if (sigma == 1) { *optN = 0; if (relax_out) *relax_out = 0.0; return OMP_OK; }

    int64_t *stride = malloc(sizeof(int64_t) * K);
    if (!stride) return OMP_ENOMEM;
    stride[K - 1] = 1;
    for (int32_t i = K - 2; i >= 0; i--) stride[i] = stride[i + 1] * (N[i + 1] + 1);

    /* C(T): every s != 0 with 0 <= s <= N and sum s_i r_i <= T,
     * by a digit odometer over the box [0, N]. */
    int64_t ncap = 64, nc = 0;
    int32_t *C = malloc(sizeof(int32_t) * ncap * K);
    int32_t *s = calloc(K, sizeof(int32_t));
    if (!C || !s) return OMP_ENOMEM;
    for (;;) {
        int32_t i = K - 1;
        while (i >= 0 && s[i] == N[i]) { s[i] = 0; i--; }
        if (i < 0) break;
        s[i]++;
        int64_t w = 0;
        for (int32_t q = 0; q < K; q++) w += (int64_t)s[q] * r[q];
        if (w > T) continue;
        if (nc == ncap) {
            ncap *= 2;
            int32_t *C2 = realloc(C, sizeof(int32_t) * ncap * K);
            if (!C2) return OMP_ENOMEM;
            C = C2;
        }
        for (int32_t q = 0; q < K; q++) C[nc * K + q] = s[q];
        nc++;
    }
    int64_t *off = malloc(sizeof(int64_t) * (nc > 0 ? nc : 1));
    if (!off) return OMP_ENOMEM;
    for (int64_t c = 0; c < nc; c++) {
        off[c] = 0;
        for (int32_t q = 0; q < K; q++) off[c] += (int64_t)C[c * K + q] * stride[q];
    }

    /* l.4–8: level of every entry; entries of each level gathered in
     * ascending index (counting sort on d). */
    int32_t *d = malloc(sizeof(int32_t) * sigma);
    int64_t *start = calloc((size_t)levels + 2, sizeof(int64_t));
    int64_t *order = malloc(sizeof(int64_t) * sigma);
    if (!d || !start || !order) return OMP_ENOMEM;
    #pragma omp parallel for schedule(static)
    for (int64_t idx = 0; idx < sigma; idx++) {
        int64_t rem = idx;
        int32_t sum = 0;
        for (int32_t q = 0; q < K; q++) { sum += (int32_t)(rem / stride[q]); rem %= stride[q]; }
        d[idx] = sum;
    }
    for (int64_t idx = 0; idx < sigma; idx++) start[d[idx] + 1]++;
    for (int32_t l = 0; l <= levels; l++) start[l + 1] += start[l];
    {
        int64_t *fill = malloc(sizeof(int64_t) * ((size_t)levels + 1));
        if (!fill) return OMP_ENOMEM;
        for (int32_t l = 0; l <= levels; l++) fill[l] = start[l];
        for (int64_t idx = 0; idx < sigma; idx++) order[fill[d[idx]]++] = idx;
        free(fill);
    }

    /* l.10–25: level by level, states of one level in parallel. */
    double relax = 0.0;
    for (int32_t l = 1; l <= levels; l++) {
        #pragma omp parallel for schedule(dynamic, 256) reduction(+:relax)
        for (int64_t t = start[l]; t < start[l + 1]; t++) {
            int64_t idx = order[t];
            int32_t v[64];
            int64_t rem = idx;
            for (int32_t q = 0; q < K; q++) { v[q] = (int32_t)(rem / stride[q]); rem %= stride[q]; }
            int32_t best = INT32_MAX;
            for (int64_t c = 0; c < nc; c++) {
                int ok = 1;
                for (int32_t q = 0; q < K; q++)
                    if (C[c * K + q] > v[q]) { ok = 0; break; }
                if (!ok) continue;
                relax += 1.0;
                int32_t o = table[idx - off[c]];
                if (o < best) best = o;
            }
            table[idx] = best + 1;
        }
    }
    *optN = table[sigma - 1];
    if (relax_out) *relax_out = relax;
    free(stride); free(C); free(s); free(off); free(d); free(start); free(order);
    return OMP_OK;
}
