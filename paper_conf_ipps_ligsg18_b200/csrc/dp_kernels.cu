// dp_kernels.cu — hand-written sm_100a kernels of the PTAS hot path.
//
//  enum_configs_kernel   §8(a) a-3: C(T) (Alg 2 l.17), once per T
//  exclusive_scan_kernel compaction offsets for a-3
//  build_prefix_kernel   a-3: group C by leading digits, packed words, off(s'),
//                        pivot blocks (D13), closed-form relaxation counts
//  row_fill_kernel       a-5: Eq. 1 for one row-level (scalar
//                        fallback: full relaxation incl. the in-row terms)
//  row_cross_kernel      a-5 for rows longer than 1 KiB (D5, D12, D13; one launch)
//  row_scatter_kernel    §8(e): gathered compact rows -> mixed-radix table
//  build_row_index_kernel a-4: level-ordered row index (row base + packed digits)
//  traceback_kernel      a-8: schedule of the rounded long jobs from DP(T*)
//
// Integer-only; no tensor cores (the DP is a min over gathers, not a
// contraction).  See DESIGN.md for the roofline of each kernel.
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "internal.h"
#include "device_common.cuh"

namespace ptas {

thread_local int64_t tl_np_hint = -1;

static std::atomic<uint64_t> g_knob_gen{1};
uint64_t knob_generation() { return g_knob_gen.load(std::memory_order_acquire); }
void knobs_refresh() { g_knob_gen.fetch_add(1, std::memory_order_acq_rel); }


namespace {

// ------------------------------------------------------------------ a-3
// One thread per prefix over the first D internal dims (mixed radix, first
// digit most significant, so thread order = lexicographic order).  Each
// thread walks its completions over dims D..K-1 in lexicographic order: the
// successor of a feasible s increments the rightmost digit d that can grow
// (s_d < hi_d and sum_{i<=d} s_i r_i + r_d <= T) and zeroes the suffix.
__global__ void enum_configs_kernel(int pass, int K, int D, int64_t nprefix,
                                    const int32_t *__restrict__ hi, const int64_t *__restrict__ r,
                                    int64_t T, const int64_t *__restrict__ stride,
                                    int64_t *__restrict__ counts, const int64_t *__restrict__ offsets,
                                    uint16_t *__restrict__ digits, int64_t *__restrict__ off, int64_t cap)
{
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nprefix) return;
    if (pass == 1 && offsets[nprefix] > cap) return;   // buffers too small: build_prefix flags it
    int32_t s[MAXK];
    uint64_t load = 0;
    bool over = false;
    int64_t rem = t;
    for (int i = D - 1; i >= 0; --i) {
        int64_t radix = (int64_t)hi[i] + 1;
        s[i] = (int32_t)(rem % radix);
        rem /= radix;
    }
    for (int i = 0; i < D; ++i) {
        load += (uint64_t)s[i] * (uint64_t)r[i];
        if (load > (uint64_t)T) over = true;
    }
    for (int i = D; i < K; ++i) s[i] = 0;
    int64_t cnt = 0;
    int64_t pos = (pass == 1) ? offsets[t] : 0;
    if (!over) {
        for (;;) {
            bool nonzero = false;
            for (int i = 0; i < K; ++i) nonzero |= (s[i] != 0);
            if (nonzero) {
                if (pass == 1) {
                    int64_t o = 0;
                    for (int i = 0; i < K; ++i) {
                        digits[(pos + cnt) * K + i] = (uint16_t)s[i];
                        o += (int64_t)s[i] * stride[i];
                    }
                    off[pos + cnt] = o;
                }
                ++cnt;
            }
            // successor over dims D..K-1
            uint64_t pl = load;   // sum_{i<=d} s_i r_i while scanning d downwards
            int d = K - 1;
            for (; d >= D; --d) {
                if (s[d] < hi[d] && pl + (uint64_t)r[d] <= (uint64_t)T) break;
                pl -= (uint64_t)s[d] * (uint64_t)r[d];
            }
            if (d < D) break;
            s[d] += 1;
            for (int i = d + 1; i < K; ++i) s[i] = 0;
            load = pl + (uint64_t)r[d];
        }
    }
    if (pass == 0) counts[t] = cnt;
}

// Single-block exclusive scan of int64 (n up to a few 1e5; planning only).
__global__ void exclusive_scan_kernel(const int64_t *__restrict__ in, int64_t *__restrict__ out,
                                      int64_t n, int64_t *__restrict__ total)
{
    __shared__ int64_t warp_sums[32];
    __shared__ int64_t carry;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    if (tid == 0) carry = 0;
    __syncthreads();
    for (int64_t base = 0; base < n; base += blockDim.x) {
        int64_t i = base + tid;
        int64_t v = i < n ? in[i] : 0;
        int64_t x = v;
        for (int o = 1; o < 32; o <<= 1) {
            int64_t y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) warp_sums[wid] = x;
        __syncthreads();
        if (wid == 0) {
            int64_t w = lane < (int)(blockDim.x >> 5) ? warp_sums[lane] : 0;
            for (int o = 1; o < 32; o <<= 1) {
                int64_t y = __shfl_up_sync(FULL, w, o);
                if (lane >= o) w += y;
            }
            warp_sums[lane] = w;
        }
        __syncthreads();
        int64_t incl = x + (wid > 0 ? warp_sums[wid - 1] : 0) + carry;
        if (i < n) out[i] = incl - v;
        __syncthreads();
        if (tid == blockDim.x - 1) carry = incl;
        __syncthreads();
    }
    if (tid == 0) *total = carry;
}

// ------------------------------------------------------------------ a-3 grouping
__device__ __forceinline__ bool same_lead(const uint16_t *a, const uint16_t *b, int K1)
{
    for (int i = 0; i < K1; ++i)
        if (a[i] != b[i]) return false;
    return true;
}

struct NallArg { int32_t v[MAXK]; };

__global__ void build_prefix_kernel(int K, const uint16_t *__restrict__ digits,
                                    const int64_t *__restrict__ off, const int64_t *__restrict__ d_nC,
                                    int64_t nc_cap, int64_t np_cap, RowGeom g,
                                    NallArg Nall, PrefixEntry *__restrict__ pref,
                                    DpMeta *__restrict__ meta)
{
    const int64_t nC = *d_nC;
    if (nC > nc_cap) {   // uniform: the buffers were sized for nc_cap configurations
        if (threadIdx.x == 0) {
            meta->nC = nC;
            meta->nP = 0;
            meta->ovf = 1;
        }
        return;
    }
    __shared__ int64_t warp_sums[32];
    __shared__ int64_t carry;
    __shared__ unsigned long long relax_acc, exec_acc;
    __shared__ int32_t blo[MAXK], bhi[MAXK];   // pivot blocks (D13), nonzero-prefix indices
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int K1 = K - 1;
    if (tid == 0) { carry = 0; relax_acc = 0ull; exec_acc = 0ull; }
    if (tid < MAXK) { blo[tid] = INT32_MAX; bhi[tid] = -1; }
    __syncthreads();
    unsigned long long my_relax = 0, my_exec = 0;
    for (int64_t base = 0; base < nC; base += blockDim.x) {
        int64_t c = base + tid;
        bool valid = c < nC;
        const uint16_t *dc = digits + c * K;
        bool head = valid && (c == 0 || !same_lead(dc, dc - K, K1));
        int64_t v = head ? 1 : 0;
        int64_t x = v;
        for (int o = 1; o < 32; o <<= 1) {
            int64_t y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) warp_sums[wid] = x;
        __syncthreads();
        if (wid == 0) {
            int64_t w = lane < (int)(blockDim.x >> 5) ? warp_sums[lane] : 0;
            for (int o = 1; o < 32; o <<= 1) {
                int64_t y = __shfl_up_sync(FULL, w, o);
                if (lane >= o) w += y;
            }
            warp_sums[lane] = w;
        }
        __syncthreads();
        int64_t incl = x + (wid > 0 ? warp_sums[wid - 1] : 0) + carry;
        if (valid) {
            int64_t id = incl - 1;
            if (head) {
                PrefixEntry e;
                for (int w = 0; w < MAXW; ++w) e.w[w] = 0;
                int64_t o = 0;
                for (int i = 0; i < K1; ++i) {
                    e.w[g.word[i]] |= (uint64_t)dc[i] << g.shift[i];
                    o += (int64_t)dc[i] * g.stride[i];
                }
                e.off = o;
                e.jmax = 0;
                e.pad = 0;
                pref[id] = e;
                // executed window gathers (D5, D12, D13): one per (row p >= s' whose first
                // nonzero digit is q = fnz(s'), x) for s' != 0; none for s' = 0 (the
                // in-row configurations never win for p != 0; row 0 is a closed form)
                int q = 0;
                while (q < K1 && dc[q] == 0) ++q;
                if (q < K1) {
                    unsigned long long rows_piv = 1;
                    for (int i = q; i < K1; ++i) rows_piv *= (unsigned long long)(Nall.v[i] - dc[i] + 1);
                    const unsigned long long Wl = (unsigned long long)Nall.v[K - 1] + 1;
                    my_exec += rows_piv * Wl;
                    atomicMin(&blo[q], (int32_t)(id - 1));   // index in the nonzero-prefix list
                    atomicMax(&bhi[q], (int32_t)(id - 1));
                }
            }
            // closed-form relaxation count: prod_i (N_i - s_i + 1) states dominate s
            unsigned long long pr = 1;
            for (int i = 0; i < K; ++i) pr *= (unsigned long long)(Nall.v[i] - dc[i] + 1);
            my_relax += pr;
        }
        __syncthreads();
        if (valid) {
            bool tail = (c == nC - 1) || !same_lead(dc, dc + K, K1);
            if (tail) pref[incl - 1].jmax = dc[K - 1];
        }
        if (tid == blockDim.x - 1) carry = incl;
        __syncthreads();
    }
    atomicAdd(&relax_acc, my_relax);
    atomicAdd(&exec_acc, my_exec);
    __syncthreads();
    if (tid == 0) {
        meta->nC = nC;
        meta->nP = carry;
        meta->relax = relax_acc;
        meta->relax_exec = exec_acc;
        meta->ovf = carry - 1 > np_cap ? 1 : 0;
    }
    // pivot blocks: [first, last + 1) per first-nonzero digit, empty = [0, 0)
    if (tid < MAXK && g.blk) {
        const bool ne = tid < K1 && bhi[tid] >= 0;
        g.blk[2 * tid] = ne ? blo[tid] : 0;
        g.blk[2 * tid + 1] = ne ? bhi[tid] + 1 : 0;
    }
}

// ------------------------------------------------------------------ a-4
// Level-ordered row index (the materialised order[] of SURVEY.md §8(a) a-4):
// thread t finds its row-level rho by binary search in level_start (prefix
// sums of the row counts = coefficients of prod_{i<K-1} (1+z+...+z^{N_i})),
// unranks slot t - level_start[rho] within the level (lexicographic order)
// with the suffix-count table, and stores the row base index and the packed
// leading digits used by the dominance test.
template <int NW>
__global__ void build_row_index_kernel(const RowGeom g, const int64_t *__restrict__ cnt_g,
                                       const int64_t *__restrict__ level_start_g, int64_t rows,
                                       int64_t *__restrict__ rb, uint64_t *__restrict__ pw, int R,
                                       int tables_in_smem)
{
    // Each thread produces R consecutive slots: one unranking (binary search +
    // suffix-count walk), then the lexicographic successor within the level.
    // Results are staged in shared memory and written out coalesced; the
    // suffix-count table and level_start are staged too when they fit.
    extern __shared__ int64_t s_tab[];
    const int ld = g.rho_max + 1;
    const int64_t ncnt = (int64_t)(g.K1 + 1) * ld;
    const int64_t *cnt = cnt_g, *level_start = level_start_g;
    int64_t *s_out = s_tab + (tables_in_smem ? ncnt + ld + 1 : 0);   // [R * blockDim][1 + NW]
    if (tables_in_smem) {
        for (int64_t i = threadIdx.x; i < ncnt + ld + 1; i += blockDim.x)
            s_tab[i] = i < ncnt ? cnt_g[i] : level_start_g[i - ncnt];
        __syncthreads();
        cnt = s_tab;
        level_start = s_tab + ncnt;
    }
    const int64_t span = (int64_t)R * blockDim.x;
    const int64_t b0 = (int64_t)blockIdx.x * span;
    const int64_t t0 = b0 + (int64_t)threadIdx.x * R;
    if (t0 < rows) {
        int lo = 0, hi = g.rho_max;  // largest rho with level_start[rho] <= t0
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (level_start[mid] <= t0) lo = mid;
            else hi = mid - 1;
        }
        int32_t d[MAXK];
        unrank_digits(g, cnt, lo, t0 - level_start[lo], d);
        int64_t next_level = level_start[lo + 1];
        const int64_t tend = t0 + R < rows ? t0 + R : rows;
        for (int64_t t = t0; t < tend; ++t) {
            if (t == next_level) {   // first row of the next level
                ++lo;
                unrank_digits(g, cnt, lo, 0, d);
                next_level = level_start[lo + 1];
            }
            int64_t base = 0;
            uint64_t w[NW];
#pragma unroll
            for (int q = 0; q < NW; ++q) w[q] = 0;
            for (int i = 0; i < g.K1; ++i) {
                base += (int64_t)d[i] * g.stride[i];
#pragma unroll
                for (int q = 0; q < NW; ++q)
                    if (g.word[i] == q) w[q] |= (uint64_t)d[i] << g.shift[i];
            }
            const int64_t k = t - b0;
            s_out[k] = base;
#pragma unroll
            for (int q = 0; q < NW; ++q) s_out[(q + 1) * span + k] = (int64_t)w[q];
            if (t + 1 < next_level) next_in_level(g, d);
        }
    }
    __syncthreads();
    const int64_t n = rows - b0 < span ? rows - b0 : span;
    for (int64_t k = threadIdx.x; k < n; k += blockDim.x) {
        rb[b0 + k] = s_out[k];
#pragma unroll
        for (int q = 0; q < NW; ++q) pw[(int64_t)q * rows + b0 + k] = (uint64_t)s_out[(q + 1) * span + k];
    }
}

// ------------------------------------------------------------------ a-5
// Scalar level fill of one row-level (Eq. 1); the fallback of
// the packed-word kernel (rows longer than 1 KiB, very large shifts).  A lane
// group of Wg = 2^wlog lanes owns one row p (32/Wg rows per warp); lanes
// cover x in chunks of Wg.  For each state n = (p, x):
//   acc(x) = min over prefixes s' != 0 with s' <= p and j in
//            [0, min(Jmax(s'), x)] of OPT(p - s', x - j)   (cross-row relaxations)
//   OPT(p, x) = 1 + min(acc(x), min_{1<=j<=min(J0,x)} OPT(p, x - j))
// Dominance s' <= p is a packed-digit compare ((P|G) - S') & G == G done
// cooperatively: lane xl tests prefix base+xl and a ballot yields the group's
// dominated set.  The row base and packed digits come from the row index.
template <typename E, int NW, bool MULTI>
__global__ void __launch_bounds__(256)
row_fill_kernel(E *table, const RowGeom g, const int64_t *__restrict__ rb, const uint64_t *__restrict__ pwa,
                int64_t pw_stride, const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta,
                int J0, int rho, int64_t slot_begin, int64_t slot_count, E *compact, int wlog)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    if (meta->ovf) return;   // enumeration overflowed its bounds: the host redoes the DP
    const int np = (int)(meta->nP - 1);      // cross-row prefixes (entry 0 is s' = 0)
    uint64_t *s_oj = reinterpret_cast<uint64_t *>(smem_raw);
    uint64_t *s_w = s_oj + np;
    for (int i = threadIdx.x; i < np; i += blockDim.x) {
        const PrefixEntry pe = gpref[1 + i];
        s_oj[i] = ((uint64_t)(uint32_t)pe.jmax << 48) | (uint64_t)pe.off;
#pragma unroll
        for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = pe.w[w];
    }
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int Wg = 1 << wlog;
    const int grp = lane >> wlog;
    const int xl = lane & (Wg - 1);
    const int rpw = 32 >> wlog;
    const unsigned gmask = Wg == 32 ? 0xffffffffu : ((1u << Wg) - 1u);
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t W = g.W;
    uint64_t guard[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) guard[w] = g.guard[w];

    for (int64_t sb = gw * rpw; sb < slot_count; sb += nw * rpw) {
        const int64_t slot = sb + grp;
        const bool rowok = slot < slot_count;
        int64_t rowbase = 0;
        uint64_t pw[NW];
#pragma unroll
        for (int w = 0; w < NW; ++w) pw[w] = rowok ? pwa[(int64_t)w * pw_stride + slot_begin + slot] : 0;
        if (rowok) rowbase = rb[slot_begin + slot];
        bool row0 = rowok;   // p = 0 (all leading digits zero): OPT(0) = 0
#pragma unroll
        for (int w = 0; w < NW; ++w) row0 &= pw[w] == 0;
        E *out = compact ? compact + slot * g.Wp : table + rowbase;
        for (int64_t x0 = 0; x0 < W; x0 += Wg) {
            const int64_t x = x0 + xl;
            const bool act = rowok && x < W;
            const E *rowp = table + (rowbase + x);
            int acc = INF;
            for (int base = 0; base < np; base += Wg) {
                const int c = base + xl;
                bool dom = false;
                if (rowok && c < np) {
                    dom = true;
#pragma unroll
                    for (int w = 0; w < NW; ++w)
                        dom &= (((pw[w] | guard[w]) - s_w[(size_t)w * np + c]) & guard[w]) == guard[w];
                }
                unsigned m = (__ballot_sync(FULL, dom) >> (grp << wlog)) & gmask;
                // 4 dominated prefixes at a time; lane xl loads OPT(p - s', x) (and, for
                // rows longer than a chunk, OPT(p - s', x - Wg)); x - j arrives by
                // shuffle from lane xl - j (source lane t sends v0 if t + j < Wg, else vprev)
                while (__any_sync(FULL, m != 0)) {
                    int v0[4], vp[4], jm[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        v0[q] = INF;
                        vp[q] = INF;
                        jm[q] = -1;
                        if (m) {
                            const int b = __ffs(m) - 1;
                            m &= m - 1;
                            const uint64_t oj = s_oj[base + b];
                            const E *src = rowp - (int64_t)(oj & 0xffffffffffffull);
                            jm[q] = (int)(oj >> 48);
                            if (act) v0[q] = src[0];
                            if (MULTI && x0 > 0 && xl + jm[q] >= Wg) vp[q] = src[-Wg];
                        }
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        acc = v0[q] < acc ? v0[q] : acc;
                        const int jmq = jm[q];
                        int jmax_w = jmq;
                        for (int o = 16; o >= Wg; o >>= 1) {
                            int t = __shfl_xor_sync(FULL, jmax_w, o);
                            jmax_w = t > jmax_w ? t : jmax_w;
                        }
                        for (int j = 1; j <= jmax_w; ++j) {
                            const int send = (xl + j < Wg) ? v0[q] : vp[q];
                            const int t = __shfl_sync(FULL, send, (xl - j) & (Wg - 1), Wg);
                            if (j <= jmq && t < acc) acc = t;
                        }
                    }
                }
            }
            if (act) {
                // in-row terms that reach back into earlier (stored) chunks
                const int jlim = J0 < x ? J0 : (int)x;
                for (int j = xl + 1; j <= jlim; ++j) {
                    int v = out[x - j];
                    acc = v < acc ? v : acc;
                }
            }
            int opt = (row0 && x == 0) ? 0 : acc + 1;
            // in-chunk chain: Bellman-Ford over shuffles
            const int jin = J0 < Wg - 1 ? J0 : Wg - 1;
            bool changed = jin > 0;
            while (__any_sync(FULL, changed)) {
                int nopt = opt;
                for (int j = 1; j <= jin; ++j) {
                    int v = __shfl_up_sync(FULL, opt, j, Wg);
                    if (xl >= j && v + 1 < nopt) nopt = v + 1;
                }
                changed = nopt < opt;
                opt = nopt;
            }
            if (act) out[x] = (E)opt;
            __syncwarp();
        }
    }
}

// Long rows (W > 1 KiB, beyond the packed kernel's one-row-per-group layout):
// one launch per row-level, one warp per (row, CROSS_CPT chunks of 32 entries),
// so a long row is spread over many warps.  For a row p != 0
//   OPT(p, x) = 1 + min over prefixes s' <= p of the row's pivot block of
//               OPT(p - s', x - min(x, Jmax(s')))
// (window minimum of reading D5: OPT is monotone in x; pivot block and no
// in-row term by readings D12/D13); row p = 0 is the closed form
// OPT(0, x) = ceil(x / J0).  Executed relaxations equal the packed kernel's.
constexpr int CROSS_CPT = 4;     // 32-entry chunks of one row per task

// first nonzero leading digit of a row from its packed digits (-1: p = 0)
template <int NW>
__device__ __forceinline__ int pivot_digit(const RowGeom &g, const uint64_t *pw)
{
    int wd = -1, bit = 0;
#pragma unroll
    for (int w = NW - 1; w >= 0; --w)
        if (pw[w]) {
            wd = w;
            bit = __ffsll((long long)pw[w]) - 1;
        }
    if (wd < 0) return -1;
    int q = -1;
    for (int i = 0; i < g.K1; ++i)
        if (g.word[i] == wd && g.shift[i] <= bit) q = i;
    return q;
}

template <typename E, int NW>
__global__ void __launch_bounds__(256)
row_cross_kernel(E *table, const RowGeom g, const int64_t *__restrict__ rb, const uint64_t *__restrict__ pwa,
                 int64_t pw_stride, const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta,
                 int64_t slot_count, int64_t nch, int J0)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    if (meta->ovf) return;
    const int np = (int)(meta->nP - 1);
    uint64_t *s_oj = reinterpret_cast<uint64_t *>(smem_raw);
    uint64_t *s_w = s_oj + np;
    for (int i = threadIdx.x; i < np; i += blockDim.x) {
        const PrefixEntry pe = gpref[1 + i];
        s_oj[i] = ((uint64_t)(uint32_t)pe.jmax << 48) | (uint64_t)pe.off;
#pragma unroll
        for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = pe.w[w];
    }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    uint64_t guard[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) guard[w] = g.guard[w];
    const int64_t ngrp = (nch + CROSS_CPT - 1) / CROSS_CPT;   // CROSS_CPT chunks of one row per task
    for (int64_t task = gw; task < slot_count * ngrp; task += nw) {
        const int64_t slot = task / ngrp;
        const int64_t xg = (task - slot * ngrp) * (32 * CROSS_CPT);
        uint64_t pw[NW];
#pragma unroll
        for (int w = 0; w < NW; ++w) pw[w] = pwa[(int64_t)w * pw_stride + slot];
        const int64_t rowbase = rb[slot];
        const int q = pivot_digit<NW>(g, pw);
        if (q < 0) {   // row p = 0
#pragma unroll
            for (int c = 0; c < CROSS_CPT; ++c) {
                const int64_t x = xg + 32 * c + lane;
                if (x < g.W) table[rowbase + x] = (E)((x + J0 - 1) / J0);
            }
            continue;
        }
        const int plo = g.blk[2 * q], phi = g.blk[2 * q + 1];
        const E *rowp = table + rowbase + xg + lane;
        int acc[CROSS_CPT];
#pragma unroll
        for (int c = 0; c < CROSS_CPT; ++c) acc[c] = INF;
        for (int base = plo & ~31; base < phi; base += 32) {
            const int cc = base + lane;
            bool dom = cc >= plo && cc < phi;
            if (dom) {
#pragma unroll
                for (int w = 0; w < NW; ++w)
                    dom &= (((pw[w] | guard[w]) - s_w[(size_t)w * np + cc]) & guard[w]) == guard[w];
            }
            unsigned m = __ballot_sync(FULL, dom);
            while (m) {
                const int b = __ffs(m) - 1;
                m &= m - 1;
                const uint64_t oj = s_oj[base + b];
                const int64_t jm = (int64_t)(oj >> 48);
                const int64_t off = (int64_t)(oj & 0xffffffffffffull);
                int v[CROSS_CPT];
#pragma unroll
                for (int c = 0; c < CROSS_CPT; ++c) {
                    const int64_t x = xg + 32 * c + lane;
                    const int64_t J = jm < x ? jm : x;
                    v[c] = x < g.W ? (int)rowp[32 * c - off - J] : INF;
                }
#pragma unroll
                for (int c = 0; c < CROSS_CPT; ++c) acc[c] = v[c] < acc[c] ? v[c] : acc[c];
            }
        }
#pragma unroll
        for (int c = 0; c < CROSS_CPT; ++c) {
            const int64_t x = xg + 32 * c + lane;
            if (x < g.W) table[rowbase + x] = (E)(acc[c] + 1);
        }
    }
}

// §8(e): write gathered compact rows (slot-major, pitch Wp) into the table.
template <typename E>
__global__ void __launch_bounds__(256)
row_scatter_kernel(E *__restrict__ table, const RowGeom g, const int64_t *__restrict__ rb, int64_t slot_count,
                   const E *__restrict__ compact)
{
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t slot = gw; slot < slot_count; slot += nw) {
        const int64_t rowbase = rb[slot];
        for (int64_t x = lane; x < g.Wp; x += 32) table[rowbase + x] = compact[slot * g.Wp + x];
    }
}

// §8(f)-2ii: the inverse -- rows of the table (row bases rb) into compact
// slot-major rows (pitch Wp), the halo of one chunk before ncclSend.
template <typename E>
__global__ void __launch_bounds__(256)
row_gather_kernel(const E *__restrict__ table, const RowGeom g, const int64_t *__restrict__ rb, int64_t slot_count,
                  E *__restrict__ compact)
{
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t slot = gw; slot < slot_count; slot += nw) {
        const int64_t rowbase = rb[slot];
        for (int64_t x = lane; x < g.Wp; x += 32) compact[slot * g.Wp + x] = table[rowbase + x];
    }
}

template <typename E>
__global__ void read_opt_kernel(const E *__restrict__ table, int64_t idx, DpMeta *meta)
{
    meta->opt = (int32_t)table[idx];
}

// ------------------------------------------------------------------ a-8
// Traceback (reading R11): from n = N, repeatedly take the configuration of
// smallest canonical rank with s <= n and OPT(n - s) = OPT(n) - 1.
template <typename E>
__global__ void __launch_bounds__(256)
traceback_kernel(const E *__restrict__ table, int K, const int32_t *__restrict__ N,
                 const int64_t *__restrict__ stride, const uint16_t *__restrict__ digits,
                 const int64_t *__restrict__ off, const int32_t *__restrict__ rank, int64_t nC,
                 int64_t idx_start, int32_t *__restrict__ out, int32_t max_out, int32_t *__restrict__ len,
                 DpMeta *meta)
{
    __shared__ int32_t cur[MAXK];
    __shared__ int64_t idx;
    __shared__ unsigned long long best;
    __shared__ int32_t mu;
    const int tid = threadIdx.x;
    if (tid < K) cur[tid] = N[tid];
    if (tid == 0) { idx = idx_start; mu = 0; }
    __syncthreads();
    while (idx != 0) {
        if (tid == 0) best = ~0ull;
        __syncthreads();
        const int v = (int)table[idx];
        unsigned long long mine = ~0ull;
        for (int64_t c = tid; c < nC; c += blockDim.x) {
            bool dom = true;
            for (int i = 0; i < K; ++i) dom &= digits[c * K + i] <= cur[i];
            if (dom && (int)table[idx - off[c]] == v - 1) {
                unsigned long long key = ((unsigned long long)(uint32_t)rank[c] << 32) | (uint32_t)c;
                mine = key < mine ? key : mine;
            }
        }
        atomicMin(&best, mine);
        __syncthreads();
        if (tid == 0) {
            if (best == ~0ull || mu >= max_out) {
                meta->err = 1;
                idx = 0;
            } else {
                int64_t c = (int64_t)(best & 0xffffffffull);
                out[mu++] = (int32_t)c;
                idx -= off[c];
            }
        }
        __syncthreads();
        if (meta->err) break;
        if (tid < K && best != ~0ull) {
            int64_t c = (int64_t)(best & 0xffffffffull);
            cur[tid] -= digits[c * K + tid];
        }
        __syncthreads();
    }
    if (tid == 0) *len = mu;
}

// Same traceback by ONE warp with the configurations staged in shared memory:
// no block barriers and no global reads besides the two table entries per
// step (OPT(n) and OPT(n - s), issued together), so a step is about one L2
// round trip.  The canonical ranks are unique, so the warp minimum of the
// candidate ranks names exactly one configuration.
template <typename E>
__global__ void __launch_bounds__(32)
traceback_warp_kernel(const E *__restrict__ table, int K, const int32_t *__restrict__ N,
                      const uint16_t *__restrict__ digits, const int64_t *__restrict__ off,
                      const int32_t *__restrict__ rank, int nC, int64_t idx_start, int32_t *__restrict__ out,
                      int32_t max_out, int32_t *__restrict__ len, DpMeta *meta,
                      const int32_t *__restrict__ inv = nullptr, int Kc = 0, int32_t *__restrict__ out_dig = nullptr)
{
    extern __shared__ __align__(16) unsigned char tb_smem[];
    int64_t *s_off = reinterpret_cast<int64_t *>(tb_smem);
    int32_t *s_rank = reinterpret_cast<int32_t *>(s_off + nC);
    int32_t *s_cur = s_rank + nC;
    uint16_t *s_dig = reinterpret_cast<uint16_t *>(s_cur + K);
    const int lane = threadIdx.x;
    for (int c = lane; c < nC; c += 32) {
        s_off[c] = off[c];
        s_rank[c] = rank[c];
    }
    for (int i = lane; i < nC * K; i += 32) s_dig[i] = digits[i];
    for (int i = lane; i < K; i += 32) s_cur[i] = N[i];
    __syncwarp();
    int64_t idx = idx_start;
    int32_t mu = 0;
    bool err = false;
    while (idx != 0) {
        const int v = (int)table[idx];
        uint32_t bestr = 0xffffffffu;
        int bestc = -1;
        for (int c = lane; c < nC; c += 32) {
            bool dom = true;
            for (int i = 0; i < K; ++i) dom &= s_dig[c * K + i] <= s_cur[i];
            if (dom && (int)table[idx - s_off[c]] == v - 1 && (uint32_t)s_rank[c] < bestr) {
                bestr = (uint32_t)s_rank[c];
                bestc = c;
            }
        }
        const uint32_t m = __reduce_min_sync(FULL, bestr);
        if (m == 0xffffffffu || mu >= max_out) {
            err = true;
            break;
        }
        const int c = __shfl_sync(FULL, bestc, __ffs(__ballot_sync(FULL, bestr == m)) - 1);
        if (lane == 0) out[mu] = c;
        if (out_dig)   // the machine's configuration in canonical class order
            for (int j = lane; j < Kc; j += 32) out_dig[(size_t)mu * Kc + j] = inv[j] < 0 ? 0 : s_dig[c * K + inv[j]];
        ++mu;
        idx -= s_off[c];
        __syncwarp();
        for (int i = lane; i < K; i += 32) s_cur[i] -= s_dig[c * K + i];
        __syncwarp();
    }
    if (lane == 0) {
        *len = mu;
        if (err) meta->err = 1;
    }
}

// Same traceback with everything in registers (nC <= 32 G configurations, K <=
// KM classes): lane l owns configurations l, l + 32 (digits, offset, rank), the
// state n is replicated in every lane, OPT(n) is tracked instead of re-read
// (each step lowers it by exactly one), so a step is ONE table load per owned
// configuration, a min-reduction over the ranks and K shuffles of the chosen
// digits.  Same choices as the one-step kernels (reading R11).
template <typename E, int G, int KM>
__global__ void __launch_bounds__(32)
traceback_reg_kernel(const E *__restrict__ table, int K, const int32_t *__restrict__ N,
                     const uint16_t *__restrict__ digits, const int64_t *__restrict__ off,
                     const int32_t *__restrict__ rank, int nC, int64_t idx_start, int32_t *__restrict__ out,
                     int32_t max_out, int32_t *__restrict__ len, DpMeta *meta, const int32_t *__restrict__ inv,
                     int Kc, int32_t *__restrict__ out_dig)
{
    const int lane = threadIdx.x;
    int dg[G][KM];
    int64_t of[G];
    uint32_t rk[G];
#pragma unroll
    for (int g = 0; g < G; ++g) {
        const int c = lane + 32 * g;
        const bool ex = c < nC;
        of[g] = ex ? off[c] : 0;
        rk[g] = ex ? (uint32_t)rank[c] : 0xffffffffu;
#pragma unroll
        for (int i = 0; i < KM; ++i) dg[g][i] = (ex && i < K) ? (int)digits[(size_t)c * K + i] : (1 << 30);
    }
    int cur[KM];
#pragma unroll
    for (int i = 0; i < KM; ++i) cur[i] = i < K ? N[i] : (1 << 30);
    int64_t idx = idx_start;
    int v = (int)table[idx];
    int32_t mu = 0;
    bool err = false;
    while (idx != 0) {
        int val[G];
#pragma unroll
        for (int g = 0; g < G; ++g) {
            bool dom = true;
#pragma unroll
            for (int i = 0; i < KM; ++i) dom &= dg[g][i] <= cur[i];
            val[g] = dom ? (int)table[idx - of[g]] : -1;
        }
        uint32_t br = 0xffffffffu;
        int bg = 0;
#pragma unroll
        for (int g = 0; g < G; ++g)
            if (val[g] == v - 1 && rk[g] < br) {
                br = rk[g];
                bg = g;
            }
        const uint32_t m = __reduce_min_sync(FULL, br);
        if (m == 0xffffffffu || mu >= max_out) {
            err = true;
            break;
        }
        const int src = __ffs(__ballot_sync(FULL, br == m)) - 1;
        const int g_ = __shfl_sync(FULL, bg, src);
        int dd[KM];
#pragma unroll
        for (int i = 0; i < KM; ++i) {
            const int mine = G == 1 ? dg[0][i] : (bg == 1 ? dg[G - 1][i] : dg[0][i]);
            dd[i] = __shfl_sync(FULL, mine, src);
            cur[i] -= i < K ? dd[i] : 0;
        }
        const int64_t myoff = G == 1 ? of[0] : (bg == 1 ? of[G - 1] : of[0]);
        idx -= __shfl_sync(FULL, myoff, src);
        --v;
        if (lane == 0) out[mu] = src + 32 * g_;
        if (out_dig)   // the machine's configuration in canonical class order
            for (int j = lane; j < Kc; j += 32) {
                const int ij = inv[j];
                int d = 0;
#pragma unroll
                for (int i = 0; i < KM; ++i) d = i == ij ? dd[i] : d;
                out_dig[(size_t)mu * Kc + j] = d;
            }
        ++mu;
    }
    if (lane == 0) {
        *len = mu;
        if (err) meta->err = 1;
    }
}

// Canonical lexicographic rank of every configuration (reading R11): rank(c)
// = #{c' : key(c') < key(c)}, key = the digits in canonical class order
// (inv[j] = internal position of canonical class j, -1 = empty class, digit 0).
__global__ void rank_configs_kernel(const uint16_t *__restrict__ digits, int nC, int K,
                                    const int32_t *__restrict__ inv, int Kc, int32_t *__restrict__ rank)
{
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nC) return;
    int32_t rk = 0;
    for (int c2 = 0; c2 < nC; ++c2) {
        int cmp = 0;   // key(c2) vs key(c)
        for (int j = 0; j < Kc && cmp == 0; ++j) {
            const int i = inv[j];
            if (i < 0) continue;
            const int a = digits[(size_t)c2 * K + i], b = digits[(size_t)c * K + i];
            cmp = a < b ? -1 : (a > b ? 1 : 0);
        }
        rk += cmp < 0;
    }
    rank[c] = rk;
}

template <typename E>
__global__ void compact_rows_kernel(const E *__restrict__ src, E *__restrict__ dst, int64_t rows, int64_t W,
                                    int64_t Wp)
{
    const int lane = threadIdx.x & 31;
    int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (; r < rows; r += nw)
        for (int64_t x = lane; x < W; x += 32) dst[r * W + x] = src[r * Wp + x];
}

__global__ void fill_value_kernel(uint8_t *p, int64_t bytes, uint8_t v)
{
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int64_t st = (int64_t)gridDim.x * blockDim.x;
    for (; i < bytes; i += st) p[i] = v;
}

int wlog_for(int64_t W)
{
    int wlog = 0;
    while ((1 << wlog) < W && wlog < 5) ++wlog;
    return wlog;
}

}  // namespace

// ------------------------------------------------------------------ launchers
cudaError_t launch_enum_configs(int pass, int K, int D, int64_t nprefix, const int32_t *hi,
                                const int64_t *r, int64_t T, const int64_t *stride,
                                int64_t *d_counts, const int64_t *d_offsets, uint16_t *d_digits,
                                int64_t *d_off, cudaStream_t st, int64_t cap)
{
    const int bs = 128;
    int64_t blocks = (nprefix + bs - 1) / bs;
    enum_configs_kernel<<<(unsigned)blocks, bs, 0, st>>>(pass, K, D, nprefix, hi, r, T, stride,
                                                         d_counts, d_offsets, d_digits, d_off, cap);
    return cudaGetLastError();
}

cudaError_t launch_exclusive_scan(const int64_t *d_in, int64_t *d_out, int64_t n, int64_t *d_total,
                                  cudaStream_t st)
{
    exclusive_scan_kernel<<<1, 1024, 0, st>>>(d_in, d_out, n, d_total);
    return cudaGetLastError();
}

// Dominance table (D10): word c * TS + dbase[i] + v holds the bits j
// of prefix chunk c (fill-kernel prefix index 32c + j = entry 1 + 32c + j)
// whose leading digit i is <= v.  A row p dominates prefix s' iff every digit
// s'_i <= min(p_i, hi_i), so the row's mask of a chunk is the AND over i of the
// words at v = min(p_i, hi_i).
__global__ void build_dom_table_kernel(const PrefixEntry *__restrict__ pref, const DpMeta *__restrict__ meta,
                                       const RowGeom g, uint32_t *__restrict__ tab)
{
    if (meta->ovf) return;
    const int np = (int)(meta->nP - 1);
    const int nch = (np + 31) / 32;
    const int n = nch * g.TS;
    for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < n; e += gridDim.x * blockDim.x) {
        const int c = e / g.TS, r = e - c * g.TS;
        int i = 0;
        while (i + 1 < g.K1 && g.dbase[i + 1] <= r) ++i;
        const int v = r - g.dbase[i];
        const uint64_t gw = g.guard[g.word[i]] >> g.shift[i];
        const uint64_t fm = (gw & (~gw + 1)) - 1;   // bits below the field's guard bit
        uint32_t bits = 0;
        for (int j = 0; j < 32; ++j) {
            const int q = 32 * c + j;
            if (q >= np) break;
            const uint64_t d = (pref[1 + q].w[g.word[i]] >> g.shift[i]) & fm;
            if (d <= (uint64_t)v) bits |= 1u << j;
        }
        tab[e] = bits;
    }
}

cudaError_t launch_build_dom_table(const PrefixEntry *d_pref, const DpMeta *d_meta, const RowGeom &g,
                                   uint32_t *d_tab, cudaStream_t st)
{
    build_dom_table_kernel<<<4, 256, 0, st>>>(d_pref, d_meta, g, d_tab);
    return cudaGetLastError();
}

cudaError_t launch_build_prefix(int K, const uint16_t *d_digits, const int64_t *d_off, const int64_t *d_nC,
                                int64_t nc_cap, int64_t np_cap, const RowGeom &g, const int32_t *Nall,
                                PrefixEntry *d_pref, DpMeta *d_meta, cudaStream_t st)
{
    NallArg na;
    for (int i = 0; i < MAXK; ++i) na.v[i] = i < K ? Nall[i] : 0;
    build_prefix_kernel<<<1, 1024, 0, st>>>(K, d_digits, d_off, d_nC, nc_cap, np_cap, g, na, d_pref, d_meta);
    return cudaGetLastError();
}

cudaError_t launch_build_row_index(const RowGeom &g, const int64_t *d_cnt, const int64_t *d_level_start,
                                   int64_t rows, int64_t *d_rb, uint64_t *d_pw, cudaStream_t st)
{
    if (rows <= 0) return cudaSuccess;
    const int bs = 128;
    const int R = rows >= (int64_t)1 << 16 ? 8 : 1;   // slots per thread
    const int64_t threads = (rows + R - 1) / R;
    const int64_t blocks = (threads + bs - 1) / bs;
    const int NWk = g.nwords <= 1 ? 1 : 2;
    const size_t out_bytes = (size_t)R * bs * 8 * (1 + NWk);
    const size_t tab = ((size_t)(g.K1 + 1) * (g.rho_max + 1) + g.rho_max + 2) * 8;
    const int in_smem = tab + out_bytes <= 48 * 1024 ? 1 : 0;
    const size_t smem = (in_smem ? tab : 0) + out_bytes;
    if (g.nwords <= 1)
        build_row_index_kernel<1><<<(unsigned)blocks, bs, smem, st>>>(g, d_cnt, d_level_start, rows, d_rb, d_pw, R, in_smem);
    else
        build_row_index_kernel<2><<<(unsigned)blocks, bs, smem, st>>>(g, d_cnt, d_level_start, rows, d_rb, d_pw, R, in_smem);
    return cudaGetLastError();
}

cudaError_t launch_row_fill(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                            int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                            int64_t nP_bound, int J0, int rho, int64_t slot_begin, int64_t slot_count,
                            void *compact_out, int sm_count, cudaStream_t st)
{
    if (slot_count <= 0) return cudaSuccess;
    const int wlog = wlog_for(g.W);
    const int rpw = 32 >> wlog;
    const int bs = 256;
    const int64_t warps = (slot_count + rpw - 1) / rpw;
    int64_t blocks = (warps + (bs / 32) - 1) / (bs / 32);
    const int64_t cap = (int64_t)sm_count * 8;
    if (blocks > cap) blocks = cap;
    const bool MULTI = g.W > 32;
    const int NWk = g.nwords <= 1 ? 1 : 2;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    const size_t smem = (size_t)np * (8 + 8 * NWk) + 16;
    if (smem > 220 * 1024) return cudaErrorInvalidValue;
    cudaError_t err;
#define PTAS_FILL_CASE(E_, NW_, MU_)                                                              \
    do {                                                                                          \
        auto kfn = row_fill_kernel<E_, NW_, MU_>;                                                 \
        if (smem > 48 * 1024) {                                                                   \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize,          \
                                       (int)smem);                                                \
            if (err != cudaSuccess) return err;                                                   \
        }                                                                                         \
        kfn<<<(unsigned)blocks, bs, smem, st>>>((E_ *)table, g, rb, pw, pw_stride, d_pref, d_meta, \
                                                J0, rho, slot_begin, slot_count, (E_ *)compact_out, \
                                                wlog);                                            \
    } while (0)
#define PTAS_FILL_JU(E_, NW_)                                                                     \
    do {                                                                                          \
        if (MULTI) PTAS_FILL_CASE(E_, NW_, true);                                                 \
        else PTAS_FILL_CASE(E_, NW_, false);                                                      \
    } while (0)
    if (e == 1) {
        if (NWk == 1) PTAS_FILL_JU(uint8_t, 1); else PTAS_FILL_JU(uint8_t, 2);
    } else {
        if (NWk == 1) PTAS_FILL_JU(uint16_t, 1); else PTAS_FILL_JU(uint16_t, 2);
    }
#undef PTAS_FILL_JU
#undef PTAS_FILL_CASE
    return cudaGetLastError();
}

cudaError_t launch_row_fill_long(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                 int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 int sm_count, cudaStream_t st)
{
    (void)rho;
    if (slot_count <= 0) return cudaSuccess;
    const int NWk = g.nwords <= 1 ? 1 : 2;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    const size_t smem = (size_t)np * (8 + 8 * NWk) + 16;
    if (smem > 220 * 1024) return cudaErrorInvalidValue;
    const int64_t nch = (g.W + 31) / 32;
    const int bs = 256;
    const int64_t cap = (int64_t)sm_count * 8;
    int64_t blocks = (slot_count * ((nch + CROSS_CPT - 1) / CROSS_CPT) + 7) / 8;
    if (blocks > cap) blocks = cap;
    const int64_t *rbl = rb + slot_begin;
    const uint64_t *pwl = pw + slot_begin;
    cudaError_t err;
#define PTAS_LONG_CASE(E_, NW_)                                                                    \
    do {                                                                                           \
        auto kfn = row_cross_kernel<E_, NW_>;                                                      \
        if (smem > 48 * 1024) {                                                                    \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
            if (err != cudaSuccess) return err;                                                    \
        }                                                                                          \
        kfn<<<(unsigned)blocks, bs, smem, st>>>((E_ *)table, g, rbl, pwl, pw_stride, d_pref, d_meta, \
                                                slot_count, nch, J0);                              \
    } while (0)
    if (e == 1) {
        if (NWk == 1) PTAS_LONG_CASE(uint8_t, 1); else PTAS_LONG_CASE(uint8_t, 2);
    } else {
        if (NWk == 1) PTAS_LONG_CASE(uint16_t, 1); else PTAS_LONG_CASE(uint16_t, 2);
    }
#undef PTAS_LONG_CASE
    return cudaGetLastError();
}

cudaError_t launch_row_scatter(int e, void *table, const RowGeom &g, const int64_t *rb, int64_t slot_count,
                               const void *compact, int sm_count, cudaStream_t st)
{
    if (slot_count <= 0) return cudaSuccess;
    int64_t blocks = (slot_count + 7) / 8;
    const int64_t cap = (int64_t)sm_count * 8;
    if (blocks > cap) blocks = cap;
    if (e == 1)
        row_scatter_kernel<uint8_t><<<(unsigned)blocks, 256, 0, st>>>((uint8_t *)table, g, rb, slot_count, (const uint8_t *)compact);
    else
        row_scatter_kernel<uint16_t><<<(unsigned)blocks, 256, 0, st>>>((uint16_t *)table, g, rb, slot_count, (const uint16_t *)compact);
    return cudaGetLastError();
}

cudaError_t launch_row_gather(int e, const void *table, const RowGeom &g, const int64_t *rb, int64_t slot_count,
                              void *compact, int sm_count, cudaStream_t st)
{
    if (slot_count <= 0) return cudaSuccess;
    int64_t blocks = (slot_count + 7) / 8;
    const int64_t cap = (int64_t)sm_count * 8;
    if (blocks > cap) blocks = cap;
    if (e == 1)
        row_gather_kernel<uint8_t><<<(unsigned)blocks, 256, 0, st>>>((const uint8_t *)table, g, rb, slot_count, (uint8_t *)compact);
    else
        row_gather_kernel<uint16_t><<<(unsigned)blocks, 256, 0, st>>>((const uint16_t *)table, g, rb, slot_count, (uint16_t *)compact);
    return cudaGetLastError();
}

cudaError_t launch_read_opt(int e, const void *table, int64_t idx, DpMeta *d_meta, cudaStream_t st)
{
    if (e == 1) read_opt_kernel<uint8_t><<<1, 1, 0, st>>>((const uint8_t *)table, idx, d_meta);
    else read_opt_kernel<uint16_t><<<1, 1, 0, st>>>((const uint16_t *)table, idx, d_meta);
    return cudaGetLastError();
}

cudaError_t launch_traceback(int e, const void *table, int K, const int32_t *d_N,
                             const int64_t *d_stride, const uint16_t *d_digits, const int64_t *d_off,
                             const int32_t *d_rank, int64_t nC, int64_t idx_start, int32_t *d_out,
                             int32_t max_out, int32_t *d_len, DpMeta *d_meta, cudaStream_t st)
{
    // one warp with the configurations in shared memory when they fit (48 KB)
    const size_t smem = (size_t)nC * (8 + 4) + (size_t)K * 4 + (size_t)nC * K * 2 + 16;
    const int64_t tbb = PTAS_KNOB("PTAS_TB_BLOCK", 0);   // tests: 1 forces the block kernel
    if (smem <= 48 * 1024 && tbb != 1) {
        if (e == 1)
            traceback_warp_kernel<uint8_t><<<1, 32, smem, st>>>((const uint8_t *)table, K, d_N, d_digits, d_off, d_rank,
                                                                (int)nC, idx_start, d_out, max_out, d_len, d_meta);
        else
            traceback_warp_kernel<uint16_t><<<1, 32, smem, st>>>((const uint16_t *)table, K, d_N, d_digits, d_off,
                                                                 d_rank, (int)nC, idx_start, d_out, max_out, d_len,
                                                                 d_meta);
        return cudaGetLastError();
    }
    if (e == 1)
        traceback_kernel<uint8_t><<<1, 256, 0, st>>>((const uint8_t *)table, K, d_N, d_stride, d_digits, d_off, d_rank, nC, idx_start, d_out, max_out, d_len, d_meta);
    else
        traceback_kernel<uint16_t><<<1, 256, 0, st>>>((const uint16_t *)table, K, d_N, d_stride, d_digits, d_off, d_rank, nC, idx_start, d_out, max_out, d_len, d_meta);
    return cudaGetLastError();
}

cudaError_t launch_traceback_canon(int e, const void *table, int K, const int32_t *d_N, const uint16_t *d_digits,
                                   const int64_t *d_off, int32_t *d_rank, int64_t nC, const int32_t *d_inv, int Kc,
                                   int64_t idx_start, int32_t *d_out, int32_t *d_out_dig, int32_t max_out,
                                   int32_t *d_len, DpMeta *d_meta, cudaStream_t st)
{
    const size_t smem = (size_t)nC * (8 + 4) + (size_t)K * 4 + (size_t)nC * K * 2 + 16;
    if (smem > 48 * 1024 || nC > (1 << 20) || PTAS_KNOB("PTAS_TB_BLOCK", 0) == 1) return cudaErrorNotSupported;
    rank_configs_kernel<<<(unsigned)((nC + 127) / 128), 128, 0, st>>>(d_digits, (int)nC, K, d_inv, Kc, d_rank);
    // configurations and state in registers when they fit (PTAS_TB_REG=0: shared-memory warp kernel)
    if (nC <= 64 && K <= 12 && PTAS_KNOB("PTAS_TB_REG", 1) != 0) {
#define PTAS_TB_REG_GO(E_, G_, KM_)                                                                          \
    traceback_reg_kernel<E_, G_, KM_><<<1, 32, 0, st>>>((const E_ *)table, K, d_N, d_digits, d_off, d_rank, (int)nC, \
                                                        idx_start, d_out, max_out, d_len, d_meta, d_inv, Kc, d_out_dig)
        const bool g1 = nC <= 32, k8 = K <= 8;
        if (e == 1) {
            if (g1) { if (k8) PTAS_TB_REG_GO(uint8_t, 1, 8); else PTAS_TB_REG_GO(uint8_t, 1, 12); }
            else { if (k8) PTAS_TB_REG_GO(uint8_t, 2, 8); else PTAS_TB_REG_GO(uint8_t, 2, 12); }
        } else {
            if (g1) { if (k8) PTAS_TB_REG_GO(uint16_t, 1, 8); else PTAS_TB_REG_GO(uint16_t, 1, 12); }
            else { if (k8) PTAS_TB_REG_GO(uint16_t, 2, 8); else PTAS_TB_REG_GO(uint16_t, 2, 12); }
        }
#undef PTAS_TB_REG_GO
        return cudaGetLastError();
    }
    if (e == 1)
        traceback_warp_kernel<uint8_t><<<1, 32, smem, st>>>((const uint8_t *)table, K, d_N, d_digits, d_off, d_rank,
                                                            (int)nC, idx_start, d_out, max_out, d_len, d_meta, d_inv,
                                                            Kc, d_out_dig);
    else
        traceback_warp_kernel<uint16_t><<<1, 32, smem, st>>>((const uint16_t *)table, K, d_N, d_digits, d_off, d_rank,
                                                             (int)nC, idx_start, d_out, max_out, d_len, d_meta, d_inv,
                                                             Kc, d_out_dig);
    return cudaGetLastError();
}

cudaError_t launch_compact_rows(int e, const void *src, void *dst, int64_t rows, int64_t W, int64_t Wp,
                                cudaStream_t st)
{
    if (rows <= 0) return cudaSuccess;
    int64_t blocks = (rows + 7) / 8;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (e == 1) compact_rows_kernel<uint8_t><<<(unsigned)blocks, 256, 0, st>>>((const uint8_t *)src, (uint8_t *)dst, rows, W, Wp);
    else compact_rows_kernel<uint16_t><<<(unsigned)blocks, 256, 0, st>>>((const uint16_t *)src, (uint16_t *)dst, rows, W, Wp);
    return cudaGetLastError();
}

cudaError_t launch_fill_value(void *p, int64_t bytes, int value, cudaStream_t st)
{
    if (bytes <= 0) return cudaSuccess;
    int64_t blocks = (bytes + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    fill_value_kernel<<<(unsigned)blocks, 256, 0, st>>>((uint8_t *)p, bytes, (uint8_t)value);
    return cudaGetLastError();
}

}  // namespace ptas
