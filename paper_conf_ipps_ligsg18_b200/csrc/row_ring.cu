// row_ring.cu — level fill of narrow DPs on ONE thread-block cluster with the
// recent row-levels resident in distributed shared memory (§8(a) a-5; DESIGN.md
// D14).
//
// For K = 3 classes the rows are (a, b) (two leading digits, last class in the
// row) and row-level L = a + b holds at most min(N0, N1) + 1 rows, while the
// dependency chain is N0 + N1 + 1 levels long (M5s: 541 levels of <= 251
// rows).  Such a DP is bound by the latency of one level, not by bandwidth:
// through L2 with ready flags a level costs ~3.5 us (flag acquire, gathers,
// release fence, per-row tickets).  Here the C CTAs of one cluster (C = 16,
// or 8 when 16 cannot be co-scheduled) fill the DP in lockstep:
//
//   * CTA c owns the rows with a in [c A, (c + 1) A) (A = ceil((N0 + 1) / C)
//     <= 16, one row of a level per warp); the last R row-levels of its rows
//     live in a ring in its shared memory (R = 1 + the largest leading-digit
//     sum of a configuration, so every source row p - s' of level L is one of
//     levels L - R + 1 .. L - 1).  A source row (a - s0, .) is in the same CTA
//     unless a - s0 crosses the block boundary (~s0 / A of the reads): DSMEM is
//     ~20 B/cycle per SM, local shared memory ~128;
//   * a warp computes one row (a, b) of level L: for every prefix s' = (s0, s1)
//     of the row's pivot block (D13) with s' <= (a, b) it reads the source row
//     (a - s0, b - s1) from the owner CTA's ring through DSMEM
//     (local shared memory or ld.shared::cluster, ~40 / ~200 cycles instead of an L2 round trip), takes the
//     shifted window of reading D5 (shuffles + PRMT, swar_common.cuh), and
//     OPT(a, b, x) = 1 + the minimum (D12); row (0, 0) is ceil(x / J0);
//   * the row goes to the own ring slot (shared memory) and to the table in HBM
//     (the table is written once and never read back by this kernel);
//   * one cluster barrier (arrive.release / wait.acquire) per TB row-levels
//     (temporal blocking, TB = 2 by default) orders the ring writes of an
//     interval before the reads of the next: at sub-level t of an interval
//     each CTA also computes, redundantly, the (TB - 1 - t) * H rows just
//     below its block (the previous CTA's rows: same inputs, same values), so
//     every source row of the interval is in its own ring; the halo holds
//     TB * H rows per level, the ring Rdep + TB - 1 levels.
//
// Same recurrence, same windows, same executed relaxations as the packed
// kernel; the values are bit-identical (parity tests, PTAS_RING=0 for the A/B).
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <map>
#include <mutex>
#include <tuple>

#include "internal.h"
#include "swar_common.cuh"

namespace ptas {
namespace swar {
namespace {

// prefixes whose DSMEM loads are issued together (CH = 8: 4, so 32 words in flight per lane)
#ifndef PTAS_RING_PROFILE
#define PTAS_RING_PROFILE 0
#endif
// diagnostics build (-DPTAS_RING_PROFILE=1): per level, clock64 of CTA `prof_cta`
// thread 0 at level start, after its rows, after arrive, after wait
#if PTAS_RING_PROFILE
__device__ long long g_ring_prof[4][2048];
#endif

__device__ __forceinline__ uint32_t dsm_map(uint32_t local_addr, uint32_t rank)
{
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(local_addr), "r"(rank));
    return r;
}

template <int CH>
__device__ __forceinline__ Words<CH> ld_dsm(uint32_t addr)
{
    Words<CH> w;
    if constexpr (CH == 1) {
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(w.v[0]) : "r"(addr) : "memory");
    } else if constexpr (CH == 2) {
        asm volatile("ld.shared::cluster.v2.u32 {%0, %1}, [%2];" : "=r"(w.v[0]), "=r"(w.v[1]) : "r"(addr) : "memory");
    } else {
#pragma unroll
        for (int c = 0; c < CH; c += 4)
            asm volatile("ld.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];"
                         : "=r"(w.v[c]), "=r"(w.v[c + 1]), "=r"(w.v[c + 2]), "=r"(w.v[c + 3])
                         : "r"(addr + 4 * c)
                         : "memory");
    }
    return w;
}

template <int CH>
__device__ __forceinline__ void st_dsm(uint32_t addr, const Words<CH> &w)
{
    if constexpr (CH == 1) {
        asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(w.v[0]) : "memory");
    } else if constexpr (CH == 2) {
        asm volatile("st.shared::cluster.v2.u32 [%0], {%1, %2};" ::"r"(addr), "r"(w.v[0]), "r"(w.v[1]) : "memory");
    } else {
#pragma unroll
        for (int c = 0; c < CH; c += 4)
            asm volatile("st.shared::cluster.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(addr + 4 * c), "r"(w.v[c]),
                         "r"(w.v[c + 1]), "r"(w.v[c + 2]), "r"(w.v[c + 3])
                         : "memory");
    }
}

// CH consecutive words of the own CTA's ring (shared memory, 4*CH-byte aligned)
template <int CH>
__device__ __forceinline__ Words<CH> lds_words(const uint32_t *p)
{
    Words<CH> w;
    if constexpr (CH == 1) {
        w.v[0] = p[0];
    } else if constexpr (CH == 2) {
        const uint2 a = *reinterpret_cast<const uint2 *>(p);
        w.v[0] = a.x;
        w.v[1] = a.y;
    } else {
#pragma unroll
        for (int c = 0; c < CH; c += 4) {
            const uint4 a = *reinterpret_cast<const uint4 *>(p + c);
            w.v[c] = a.x;
            w.v[c + 1] = a.y;
            w.v[c + 2] = a.z;
            w.v[c + 3] = a.w;
        }
    }
    return w;
}

__device__ __forceinline__ void cluster_sync_all()
{
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Windows of one prefix for the lane's CH words: class 1 = shift of at most one
// word (db <= 4 bytes: words w - 1, w), class 2 = at most two (4 < db <= 8:
// words w - 2, w - 1); w1 / w2 = the words left of the chunk.
template <typename E, int CH, int CLS>
__device__ __forceinline__ void ring_windows(const Words<CH> &cur, uint32_t w1, uint32_t w2, uint32_t sel,
                                             Words<CH> &ae, Words<CH> &ao)
{
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const uint32_t lo = CLS == 1 ? (t == 0 ? w1 : cur.v[t - 1]) : (t >= 2 ? cur.v[t - 2] : (t == 1 ? w1 : w2));
        const uint32_t hi = CLS == 1 ? cur.v[t] : (t >= 1 ? cur.v[t - 1] : w1);
        if constexpr (sizeof(E) == 1) {
            ae.v[t] = vmin2(ae.v[t], prmt(lo, hi, sel));
            ao.v[t] = vmin2(ao.v[t], prmt(lo, hi, sel + 0x1111u));
        } else {
            ae.v[t] = vmin2(ae.v[t], prmt(lo, hi, sel));
        }
    }
}

template <typename E, int CH, int WIN>
__global__ void __launch_bounds__(1024, 1)
row_ring_kernel(E *table, const RingArgs ra, const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta)
{
    constexpr int EB = (int)sizeof(E);
    constexpr uint32_t ONES = 0x00010001u;
#ifndef PTAS_RING_PB
#define PTAS_RING_PB 4
#endif
    constexpr int PB = PTAS_RING_PB;   // prefixes whose loads are issued together
    extern __shared__ __align__(16) unsigned char smem_raw[];
    if (meta->ovf) return;   // grid-uniform: every CTA exits before any barrier
    uint32_t crank;
    asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
    const int np = (int)(meta->nP - 1);
    const int Lw = ra.Lw, Lg = ra.Lg;
    const uint32_t row_bytes = (uint32_t)Lw * 4;
    // smem: ring [R][HT + A][Lw] words (per slot: HT halo rows a0 - HT .. a0 - 1,
    // then the A own rows) | 4 prefix lists int4 [np + PB] each
    uint32_t *ring = reinterpret_cast<uint32_t *>(smem_raw);
    const int TB = ra.TB;                        // row-levels per cluster barrier
    const int HT = TB * ra.H;                    // halo rows per slot
    const int AH = ra.A + HT;
    int4 *s_pl = reinterpret_cast<int4 *>(smem_raw + (((size_t)ra.R * AH * row_bytes + 15) & ~(size_t)15));
    const int lcap = np + PB;
    __shared__ int s_cnt[4];
    if (threadIdx.x < 4) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    // prefix lists by (pivot block, window class): list 2*blk + cls - 1, blk 0 = {s0 = 0}
    // (rows a = 0), blk 1 = {s0 >= 1} (rows a >= 1); entries (s0, s1, selector | db << 16,
    // |s'|).  The order inside a list does not matter (min is commutative).
    for (int i = threadIdx.x; i < np; i += blockDim.x) {
        const PrefixEntry pe = gpref[1 + i];
        const int s0 = (int)(pe.off / ra.stride0);
        const int s1 = (int)((pe.off - (int64_t)s0 * ra.stride0) / ra.Wp);
        const int sel = oj_entry(pe, EB).y;
        const int li = 2 * (s0 >= 1) + ((sel >> 16) > 4 ? 1 : 0);
        s_pl[li * lcap + atomicAdd(&s_cnt[li], 1)] = make_int4(s0, s1, sel, s0 + s1);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * PB; i += blockDim.x)   // padding: never dominated (lists hold np + PB entries)
        s_pl[(i / PB) * lcap + s_cnt[i / PB] + i % PB] =
            make_int4(1 << 20, 1 << 20, (EB == 1 ? SEL_U8 : SEL_U16) + SEL_SELF, 0);
    uint32_t csize;
    asm("mov.u32 %0, %%cluster_nctarank;" : "=r"(csize));
    // the next CTA's ring: this CTA's top HT rows of every level are pushed into its halo
    const bool has_next = crank + 1 < csize;
    const uint32_t nxt = dsm_map((uint32_t)__cvta_generic_to_shared(ring), has_next ? crank + 1 : crank);
    __syncthreads();
    cluster_sync_all();   // every CTA of the cluster runs before any DSMEM access

    const int a0 = (int)crank * ra.A;          // first row digit a of this CTA
    uint32_t *tab32 = reinterpret_cast<uint32_t *>(table);
    int slot = 0;                              // L mod R
    Words<CH> last;
    int64_t last_off = -1;                     // word offset of the thread's last row chunk of the interval
    // TB row-levels per cluster barrier (temporal blocking): at sub-level t of an
    // interval this CTA also computes, redundantly, the (TB - 1 - t) * H rows below
    // its block (the previous CTA's rows, same values), so every source of the
    // interval's levels is either in the halo pushed before the last barrier or
    // computed here; the previous CTA's pushes of the rows computed here land in
    // the same ring positions with the same values
    for (int L0 = 0; L0 <= ra.rho_max; L0 += TB) {
#if PTAS_RING_PROFILE
        const bool pr = threadIdx.x == 0 && crank == 8 && L0 < 2048;
        if (pr) g_ring_prof[0][L0] = clock64();
#endif
        const int tn = min(TB, ra.rho_max - L0 + 1);
        for (int t = 0; t < tn; ++t) {
            const int L = L0 + t;
            const int ext = (TB - 1 - t) * ra.H;     // redundant rows below the block
            // rows of level L: a in [lo, hi] (contiguous), b = L - a
            const int lo = max(max(L - ra.N1, 0), a0 - ext);
            const int hi = min(min(L, ra.N0), a0 + ra.A - 1);
            const int ntask = hi >= lo ? (hi - lo + 1) * Lg : 0;
            for (int task = threadIdx.x; task < ntask; task += blockDim.x) {
                const int r_ = task / Lg;
                const int a = lo + r_;
                const int c = task - r_ * Lg;       // lane chunk: words c*CH .. c*CH+CH-1 of the row
                const int b = L - a;
                const int ia = a - a0;              // < 0: a redundant row of the previous CTA
                const int pos0 = (HT + ia) * Lw + c * CH;  // the lane's words within a ring slot
                Words<CH> ae, ao;
                fill_words(ae, 0xffffffffu);
                fill_words(ao, 0xffffffffu);
                const int blk = a >= 1 ? 1 : 0;    // pivot block (D13)
#pragma unroll
                for (int cls = 1; cls <= (WIN == 8 ? 2 : 1); ++cls) {
                    const int4 *pl = s_pl + (2 * blk + cls - 1) * lcap;
                    const int n = s_cnt[2 * blk + cls - 1];
                    for (int q0 = 0; q0 < n; q0 += PB) {
                        Words<CH> cur[PB];
                        uint32_t l1[PB], l2[PB];
                        int sj[PB];
#pragma unroll
                        for (int u = 0; u < PB; ++u) {
                            const int4 pf = pl[q0 + u];
                            sj[u] = pf.z;
                            // source row (a - s0, b - s1) of level L - |s'|: always in this CTA's
                            // ring (own rows, halo rows, or rows computed redundantly this interval)
                            int ss = slot - pf.w;
                            ss += ss < 0 ? ra.R : 0;
                            const int pos = pos0 + (ss * AH - pf.x) * Lw;   // word index in the ring
                            if (pf.x <= a && pf.y <= b) {
                                const uint32_t *p = ring + pos;
                                cur[u] = lds_words<CH>(p);
                                l1[u] = c >= 1 ? p[-1] : 0u;
                                l2[u] = (cls == 2 && c * CH >= 2) ? p[-2] : 0u;
                            } else {
                                fill_words(cur[u], 0xffffffffu);
                                l1[u] = l2[u] = 0xffffffffu;
                            }
                        }
#pragma unroll
                        for (int u = 0; u < PB; ++u) {
                            // positions before the row: its first entry replicated (row word 0 is
                            // the chunk's own word for c = 0, the left word for c = 1 with CH = 1)
                            uint32_t f = c == 0 ? cur[u].v[0] : l1[u];
                            f = EB == 1 ? prmt(f, 0u, 0x0000u) : prmt(f, 0u, 0x1010u);
                            const uint32_t w1 = c >= 1 ? l1[u] : f;
                            const uint32_t w2 = c * CH >= 2 ? l2[u] : f;
                            if (cls == 1) ring_windows<E, CH, 1>(cur[u], w1, w2, (uint32_t)sj[u], ae, ao);
                            else ring_windows<E, CH, 2>(cur[u], w1, w2, (uint32_t)sj[u], ae, ao);
                        }
                    }
                }
                Words<CH> wv;
#pragma unroll
                for (int t2 = 0; t2 < CH; ++t2) {
                    uint32_t oe, oo = 0;
                    if constexpr (EB == 1) {
                        oe = (ae.v[t2] & 0x00ff00ffu) + ONES;
                        oo = (ao.v[t2] & 0x00ff00ffu) + ONES;
                    } else {
                        oe = vmin2(ae.v[t2], 0xfffefffeu) + ONES;
                    }
                    if (L == 0) {   // row (0, 0): OPT(0, x) = ceil(x / J0)
                        const uint32_t x0 = (uint32_t)(c * CH + t2) * (4 / EB);
                        auto cf = [&](uint32_t x) { return (x + (uint32_t)ra.J0 - 1u) / (uint32_t)ra.J0; };
                        if constexpr (EB == 1) {
                            oe = cf(x0) | (cf(x0 + 2) << 16);
                            oo = cf(x0 + 1) | (cf(x0 + 3) << 16);
                        } else {
                            oe = cf(x0) | (cf(x0 + 1) << 16);
                        }
                    }
                    wv.v[t2] = EB == 1 ? prmt(oe, oo, 0x6240u) : oe;
                }
                store_words<CH>(ring + ((size_t)slot * AH + HT + ia) * Lw + c * CH, wv);
                if (ia >= 0) {   // own row: the halo of the next CTA, and the table in HBM
                    if (has_next && ia >= ra.A - HT)
                        st_dsm<CH>(nxt + 4u * (uint32_t)(((slot * AH + ia - (ra.A - HT)) * Lw + c * CH)), wv);
                    const int64_t off = ((int64_t)a * ra.stride0 + (int64_t)b * ra.Wp) * EB / 4 + c * CH;
                    if (t + 1 < tn || task + (int)blockDim.x < ntask) {
                        store_words<CH>(tab32 + off, wv);
                    } else {   // (the thread's last row of the interval: stored after the arrive)
                        last = wv;
                        last_off = off;
                    }
                }
            }
            slot = slot + 1 == ra.R ? 0 : slot + 1;
            if (t + 1 < tn) __syncthreads();   // level L complete in this CTA's ring
        }
        // the interval's levels complete in every CTA's ring: the release covers the ring
        // and halo stores; the thread's last row goes to HBM between arrive and wait
#if PTAS_RING_PROFILE
        if (pr) g_ring_prof[1][L0] = clock64();
#endif
        asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
#if PTAS_RING_PROFILE
        if (pr) g_ring_prof[2][L0] = clock64();
#endif
        if (last_off >= 0) store_words<CH>(tab32 + last_off, last);
        last_off = -1;
        asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
#if PTAS_RING_PROFILE
        if (pr) g_ring_prof[3][L0] = clock64();
#endif
    }
}

template <typename E, int CH, int WIN>
cudaError_t launch_ring_t(void *table, const RingArgs &ra, const PrefixEntry *d_pref, const DpMeta *d_meta,
                          int64_t nP_bound, int csize, cudaStream_t st, bool dry)
{
    auto kfn = row_ring_kernel<E, CH, WIN>;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    size_t smem = (((size_t)ra.R * (ra.A + ra.TB * ra.H) * ra.Lw * 4 + 15) & ~(size_t)15) + 4 * (size_t)(np + PTAS_RING_PB) * 16;
    if (smem > 220 * 1024) return cudaErrorNotSupported;
    // PTAS_RING_SMEM_MIN (experiment): pad the dynamic shared memory, e.g. above half an
    // SM's, so no two ring CTAs (of concurrent DPs) share an SM
    smem = std::max<size_t>(smem, (size_t)std::min<int64_t>(220 * 1024, PTAS_KNOB("PTAS_RING_SMEM_MIN", 0)));
    // function attributes and the co-residency query once per (device, kernel,
    // smem, cluster size, block): they take the driver lock, and concurrent DP
    // slots issue from several host threads
    int dev = 0;
    cudaError_t err = cudaGetDevice(&dev);
    if (err != cudaSuccess) return err;
    const int lanes = (ra.A + (ra.TB - 1) * ra.H) * ra.Lg;   // own + redundant rows of a level
    const int warps = std::min(32, (lanes + 31) / 32);
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)csize;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3((unsigned)csize);
    cfg.blockDim = dim3((unsigned)(32 * warps));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    static std::mutex mu;
    static std::map<std::tuple<int, const void *, size_t, int, int>, int> ncl_cache;
    const auto key = std::make_tuple(dev, (const void *)kfn, smem, csize, warps);
    int ncl = -1;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = ncl_cache.find(key);
        if (it != ncl_cache.end()) ncl = it->second;
    }
    if (ncl < 0) {
        err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
        if (err == cudaSuccess && csize > 8) err = cudaFuncSetAttribute(kfn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (err == cudaSuccess) err = cudaOccupancyMaxActiveClusters(&ncl, kfn, &cfg);
        if (err != cudaSuccess) {
            cudaGetLastError();
            ncl = 0;
        }
        std::lock_guard<std::mutex> lk(mu);
        ncl_cache[key] = ncl;
    }
    if (ncl < 1) return cudaErrorNotSupported;
    if (!dry && PTAS_KNOB("PTAS_TRACE", 0) == 1)
        std::fprintf(stderr, "[ring] cluster %d x %d threads, smem %zu B, slots %d (dep %d), %d levels per barrier: %d clusters co-resident\n",
                     csize, 32 * warps, smem, ra.R, ra.Rdep, ra.TB, ncl);
    if (dry) return cudaSuccess;
    err = cudaLaunchKernelEx(&cfg, kfn, (E *)table, ra, d_pref, d_meta);
#if PTAS_RING_PROFILE
    if (err == cudaSuccess) {
        static long long h[4][2048];
        cudaStreamSynchronize(st);
        cudaMemcpyFromSymbol(h, g_ring_prof, sizeof(h));
        double s0 = 0, s1 = 0, s2 = 0;
        const int nl = std::min(ra.rho_max + 1, 2048);
        int ni = 0;
        for (int L = ra.TB; L < nl; L += ra.TB, ++ni) {   // intervals of TB levels (the first skipped)
            s0 += h[1][L] - h[0][L];
            s1 += h[2][L] - h[1][L];
            s2 += h[3][L] - h[2][L];
        }
        ni = std::max(ni, 1);
        std::fprintf(stderr, "[ring] CTA 8 thread 0, cycles per interval of %d levels: rows %.0f arrive %.0f wait %.0f (levels %d, CH %d, threads %d)\n",
                     ra.TB, s0 / ni, s1 / ni, s2 / ni, nl, CH, 32 * warps);
    }
#endif
    return err;
}

template <typename E, int CH>
cudaError_t launch_ring_ch(void *table, const RingArgs &ra, const PrefixEntry *d_pref, const DpMeta *d_meta,
                           int64_t nP_bound, int csize, int win, cudaStream_t st, bool dry)
{
    if (win == 4) return launch_ring_t<E, CH, 4>(table, ra, d_pref, d_meta, nP_bound, csize, st, dry);
    return launch_ring_t<E, CH, 8>(table, ra, d_pref, d_meta, nP_bound, csize, st, dry);
}

template <typename E>
cudaError_t launch_ring_e(void *table, const RingArgs &ra, int CH, const PrefixEntry *d_pref, const DpMeta *d_meta,
                          int64_t nP_bound, int csize, int win, cudaStream_t st, bool dry)
{
    switch (CH) {
    case 1: return launch_ring_ch<E, 1>(table, ra, d_pref, d_meta, nP_bound, csize, win, st, dry);
    case 2: return launch_ring_ch<E, 2>(table, ra, d_pref, d_meta, nP_bound, csize, win, st, dry);
    case 4: return launch_ring_ch<E, 4>(table, ra, d_pref, d_meta, nP_bound, csize, win, st, dry);
    default: return launch_ring_ch<E, 8>(table, ra, d_pref, d_meta, nP_bound, csize, win, st, dry);
    }
}

}  // namespace
}  // namespace swar

// Host-side test of the ring kernel's geometry for a DP with internal counts N,
// sizes r (K classes) at T: true when launch_row_fill_ring would take it (the
// shared-memory fit for one of the cluster sizes; occupancy is not queried).
// The solve driver evaluates such latency-bound DPs concurrently (D8, D14).
bool ring_fits(const int32_t *N, const int64_t *r, int K, int64_t T)
{
    if (K != 3) return false;
    int64_t sumN = 0;
    for (int i = 0; i < K; ++i) sumN += N[i];
    const int e = sumN <= 255 ? 1 : 2;
    const int64_t W = (int64_t)N[2] + 1;
    const int Lw = (int)row_pitch_words(W * e);
    const int J0 = (int)std::min<int64_t>(N[2], T / r[2]);
    if (J0 * e > 8) return false;
    const int64_t hi0 = std::min<int64_t>(N[0], T / r[0]), hi1 = std::min<int64_t>(N[1], T / r[1]);
    const int64_t R = std::min<int64_t>(hi0 + hi1, T / std::min(r[0], r[1])) + 1;
    for (int csize : {16, 8}) {
        const int64_t A = (N[0] + csize) / csize;
        if (A < hi0) continue;
        if (((R * (A + hi0) * Lw * 4 + 15) & ~(int64_t)15) + 4 * (int64_t)(hi0 + 1) * (hi1 + 1) * 16 <= 220 * 1024)
            return true;
    }
    return false;
}

// Host planning (D14): K = 3 only (two leading digits), a row of at
// most 256 words (one warp), window shifts J0 * e <= 124 bytes, and the ring of
// R levels x A rows per CTA within the shared memory of one CTA.  Returns
// cudaErrorNotSupported when the DP does not qualify (the caller then uses the
// dataflow / per-level launches).  dry: only check (no launch).
cudaError_t launch_row_fill_ring(int e, void *table, const RowGeom &g, const int32_t *N, const int64_t *r,
                                 int64_t T, int J0, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, cudaStream_t st, bool dry)
{
    if (g.K1 != 2 || (g.Wp * e) % 4 != 0) return cudaErrorNotSupported;
    const int Lw = (int)(g.Wp * e / 4);
    // windows up to two words left (J0 * e <= 8 bytes: the M5s shapes have 6)
    if (J0 * e > 8) return cudaErrorNotSupported;
    if (PTAS_KNOB("PTAS_RING", 1) == 0) return cudaErrorNotSupported;
    RingArgs ra;
    ra.N0 = N[0];
    ra.N1 = N[1];
    ra.Wp = (int32_t)g.Wp;
    ra.stride0 = g.stride[0];
    ra.Lw = Lw;
    ra.J0 = J0;
    // ring depth: 1 + the largest leading-digit sum of a configuration, bounded by
    // min(hi0 + hi1, floor(T / min(r0, r1)))
    const int64_t hi0 = std::min<int64_t>(N[0], T / r[0]), hi1 = std::min<int64_t>(N[1], T / r[1]);
    // the prefix lists hold the distinct leading parts (s0, s1) <= (hi0, hi1): size the
    // shared memory by that, not by the engine's generic bound (which is NP_CAP when
    // the DP is enqueued without reading |C| back): a 16-CTA cluster of 1 CTA per SM
    // fits 7 times on the GPU, of 2 CTAs per SM 14 times (measured), so concurrent
    // ring DPs of a speculative chain all co-reside only with the tight size
    nP_bound = std::min<int64_t>(nP_bound, (hi0 + 1) * (hi1 + 1));
    if (nP_bound > 4096) return cudaErrorNotSupported;
    ra.Rdep = (int)std::min<int64_t>(hi0 + hi1, T / std::min(r[0], r[1])) + 1;
    ra.rho_max = N[0] + N[1];
    const int win = J0 * e <= 4 ? 4 : 8;
    const size_t smem_cap = 220 * 1024;
    // row-levels per cluster barrier (temporal blocking): up to PTAS_RING_TB, as long
    // as two CTAs still fit one SM (14 co-resident clusters, D14) and the halo
    // (TB * H rows) comes from the previous CTA's block alone
    const int tb_max = (int)std::max<int64_t>(1, PTAS_KNOB("PTAS_RING_TB", 2));
    const size_t smem_target = (size_t)PTAS_KNOB("PTAS_RING_SMEM_TARGET", 112 * 1024);
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    const int cs_force = (int)PTAS_KNOB("PTAS_RING_CS", 0);   // experiment: force the cluster size
    for (int csize : {16, 8, 4, 2}) {
        if (cs_force ? csize != cs_force : csize < 8) continue;
        ra.A = (N[0] + csize) / csize;   // ceil((N0 + 1) / C) rows of each level per CTA
        ra.H = (int32_t)hi0;              // halo rows per level (s0 <= hi0)
        if (ra.A < hi0) continue;         // every source row is in this CTA's block or the previous one
        // ring slots: the Rdep levels a row reads plus the TB - 1 levels of the interval
        auto smem_of = [&](int tb) {
            return (((size_t)(ra.Rdep + tb - 1) * (ra.A + tb * ra.H) * Lw * 4 + 15) & ~(size_t)15) +
                   4 * (size_t)(np + PTAS_RING_PB) * 16;
        };
        int TB = tb_max;
        while (TB > 1 && (ra.A < TB * ra.H || smem_of(TB) > smem_target)) --TB;
        if (smem_of(TB) > smem_cap) continue;
        ra.TB = TB;
        ra.R = ra.Rdep + TB - 1;
        const int rows_max = ra.A + (TB - 1) * ra.H;   // own + redundant rows of a level
        // words per lane: the smallest chunk with one pass over the CTA's rows of a level
        // words per lane: 4 when the CTA's rows of a level fit one pass (measured best on
        // M5s: 2 words 1.82 / 1.69 ms, 4 words 1.39 / 1.48 ms, 8 words 1.94 / 1.96 ms per DP),
        // else the smallest chunk that fits, else 8
        int CH = 8;
        if (Lw % 4 == 0 && (int64_t)rows_max * (Lw / 4) <= 1024) CH = 4;
        else
            for (int c : {1, 2, 4})
                if (Lw % c == 0 && (int64_t)rows_max * (Lw / c) <= 1024) {
                    CH = c;
                    break;
                }
        const int ch_env = (int)PTAS_KNOB("PTAS_RING_CH", 0);   // experiment knob: words per lane
        if (ch_env == 1 || ch_env == 2 || ch_env == 4 || ch_env == 8) CH = ch_env;
        if (Lw % CH != 0) continue;
        ra.Lg = Lw / CH;
        cudaError_t err = e == 1 ? swar::launch_ring_e<uint8_t>(table, ra, CH, d_pref, d_meta, nP_bound, csize, win, st, dry)
                                 : swar::launch_ring_e<uint16_t>(table, ra, CH, d_pref, d_meta, nP_bound, csize, win, st, dry);
        if (err == cudaSuccess) return err;
        cudaGetLastError();
    }
    return cudaErrorNotSupported;
}

}  // namespace ptas
