// device_common.cuh — device helpers shared by the fill kernels (product only).
#pragma once
#include <cstdint>

#include "internal.h"

namespace ptas {

constexpr unsigned FULL = 0xffffffffu;
constexpr int INF = 1 << 28;

// ------------------------------------------------------------------ a-4 (stepping)
// Digits of the rank-th row of row-level rho (lexicographic), as unrank_row.
__device__ __forceinline__ static void unrank_digits(const RowGeom &g, const int64_t *cnt, int rho, int64_t rank,
                                              int32_t *d)
{
    const int ld = g.rho_max + 1;
    int L = rho;
    for (int i = 0; i < g.K1; ++i) {
        int lo = L - g.maxsuf[i + 1];
        if (lo < 0) lo = 0;
        int hi = g.N[i] < L ? g.N[i] : L;
        int v = lo;
        const int64_t *row = cnt + (int64_t)(i + 1) * ld;
        for (; v < hi; ++v) {
            int64_t c = row[L - v];
            if (rank < c) break;
            rank -= c;
        }
        d[i] = v;
        L -= v;
    }
}

// Lexicographic successor among the vectors with the same digit sum: raise the
// rightmost digit i that can grow while some weight remains to its right, then
// give the rest of that weight to the suffix as far right as possible.
__device__ __forceinline__ static void next_in_level(const RowGeom &g, int32_t *d)
{
    const int K1 = g.K1;
    int suf = d[K1 - 1];
    int i = K1 - 2;
    for (; i >= 0; --i) {
        if (d[i] < g.N[i] && suf >= 1) break;
        suf += d[i];
    }
    if (i < 0) return;  // no successor (caller never asks past the level end)
    d[i] += 1;
    suf -= 1;
    for (int t = K1 - 1; t > i; --t) {
        int v = g.N[t] < suf ? g.N[t] : suf;
        d[t] = v;
        suf -= v;
    }
}


}  // namespace ptas
