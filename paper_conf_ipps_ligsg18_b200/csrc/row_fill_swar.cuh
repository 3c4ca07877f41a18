// row_fill_swar.cuh — packed-word level fill kernel template (see row_fill_swar.cu).
// Included by the four instantiation units row_fill_swar_<E>_nw<NW>.cu so the
// variants of each (entry type, digit words) pair compile in parallel.
#pragma once
//
// Eq. 1 of PAPER.md:74-79 on the row wavefront (row-level rho = sum of the
// K-1 leading digits p of n = (p, x)), with the result-identical reduction of
// SURVEY.md §8(f)-1 (reading D5): OPT is monotone under dominance,
// so for a prefix s' of C(T) (the leading K-1 digits of configurations s)
//
//     min_{0 <= j <= min(x, Jmax(s'))} OPT(p - s', x - j) = OPT(p - s', x - min(x, Jmax(s')))
//
// Per (row, prefix) the kernel therefore takes ONE shifted window of the
// source row instead of Jmax(s') + 1 of them.  Two more result-identical
// restrictions follow from the bins of a packing being unordered (DESIGN.md
// D12, D13): for a row p != 0 some bin of an optimal packing holds an item
// of the row's first nonzero leading class q, so only the prefixes with
// s'_q >= 1 (one contiguous block of the lexicographic prefix list) are
// walked, and the in-row configurations (0, j) never win; row p = 0 is the
// closed form OPT(0, x) = ceil(x / J0).  OPT(p, x) = 1 + the window minimum:
// no in-row closure, no chain.  Values are bit-identical to the plain
// recurrence (pinned by the parity tests).
//
// Lane layout: a row of Lw 32-bit words (pitch padded by the driver to a
// multiple of CH words) is owned by a group of Lg = Lw / CH lanes; lane xl of
// the group holds the CH consecutive words xl*CH .. xl*CH+CH-1 (one vector
// load per source row).  uint8 windows are split into even/odd uint16 lanes
// with the sign-replicating PRMT mode (v < 128 -> v, v >= 128 -> 0xFF00|v, a
// monotone encoding) so VIMNMX.U16x2 takes two minima per instruction.  All
// row groups of a warp walk the prefix list in lockstep (uniform loop,
// uniform shift), each with its own dominance mask s' <= p; a warp whose rows
// all dominate every prefix (p >= hi digit-wise, "interior") skips the mask.
// Positions x - J < 0 take the row's first entry (the clamp min(x, J)).
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <cuda_runtime.h>
#include <mutex>
#include <unordered_map>

#include "device_common.cuh"
#include "internal.h"
#include "swar_common.cuh"

namespace ptas {
namespace swar {


// Prefix offsets/Jmax in constant memory: indexed by a warp-uniform loop
// counter they load into uniform registers.  One slot per DP slot of the engine.
constexpr int CP_MAX = 1000;   // per DP slot
constexpr int CP_SLOTS = 4;
struct ConstPref {
    int np;
    int pad;
    int2 oj[CP_MAX];
};
static __constant__ ConstPref c_pref[CP_SLOTS];  // one copy per translation unit (no -rdc)

static __global__ void pack_const_prefix_kernel(const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta,
                                         int eb, ConstPref *__restrict__ out)
{
    if (meta->ovf) return;   // enumeration overflowed its bounds (the fill kernels exit too)
    const int np = (int)(meta->nP - 1);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        out->np = np;
        out->pad = 0;
    }
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ((np + 31) & ~31) && i < CP_MAX;
         i += gridDim.x * blockDim.x) {
        if (i < np) {
            const PrefixEntry pe = gpref[1 + i];
            out->oj[i] = oj_entry(pe, eb);
        } else {
            out->oj[i] = make_int2(0, (eb == 1 ? SEL_U8 : SEL_U16) + SEL_SELF);
        }
    }
}

static cudaError_t prepare_const_prefix_tu(const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound,
                                           int e, int cslot, void *d_staging, cudaStream_t st)
{
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    if (np > CP_MAX || cslot < 0 || cslot >= CP_SLOTS) return cudaErrorNotSupported;
    pack_const_prefix_kernel<<<8, 256, 0, st>>>(d_pref, d_meta, e, (ConstPref *)d_staging);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return err;
    const size_t bytes = 8 + 8 * (size_t)std::min<int64_t>((np + 31) & ~(int64_t)31, CP_MAX);   // within the slot
    return cudaMemcpyToSymbolAsync(c_pref, d_staging, bytes, (size_t)cslot * sizeof(ConstPref),
                                   cudaMemcpyDeviceToDevice, st);
}

// E: uint8_t / uint16_t entries; NW: 64-bit words of packed leading digits;
// CH: words per lane; WIN: largest prefix window shift in bytes the kernel
// supports (J0 * e <= 4, <= 8, or 0 = any);
// CPREF: prefix offsets from the constant bank; SPLIT: the warps of a block
// share rows (small row-levels with long prefix lists); DF: dataflow launch
// over a run of row-levels (D7; rho, slot_begin and slot_count
// are unused, the row sets come from df).
// Resident blocks per SM the compiler must allow (register cap 65536 / (256 * MINB)):
// uint16 tables 4 (64 registers: M3s 8.8 -> 8.1 ms, M5s-0.15 21.8 -> 20.3 ms fill,
// measured), uint8 tables 4 (64 registers, round 2: M2s 2.31 -> 2.23 ms, M4x
// 96.4 -> 94.8 ms, M4s / M3g unchanged, against 3 blocks at 80 registers; in
// round 1, before the pivot blocks, 64 spilled: M2s 3.40 -> 3.59 ms; uncapped,
// the dominance-table code takes 90-96 and 2 blocks/SM: M4s +13%).
#ifndef PTAS_MINB_U8
#define PTAS_MINB_U8 4
#endif
#ifndef PTAS_MINB_U16
#define PTAS_MINB_U16 4
#endif
template <typename E, int NW, int CH, int WIN, bool CPREF, bool SPLIT, int DFM>
__global__ void __launch_bounds__(256, sizeof(E) == 1 ? PTAS_MINB_U8 : PTAS_MINB_U16)
row_fill_swar_kernel(E *table, const RowGeom g, const int64_t *__restrict__ rb,
                     const uint64_t *__restrict__ pwa, int64_t pw_stride,
                     const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta, int J0,
                     int rho, int64_t slot_begin, int64_t slot_count, E *compact, int Lg, int nsplit_arg, int cslot,
                     const DfArgs df)
{
    constexpr int EB = (int)sizeof(E);
    constexpr uint32_t ONES = 0x00010001u;
    // DFM = 0: one row-level per launch; 1: dataflow run (tickets + ready flags,
    // DESIGN.md D7); 2: cluster run (the CTAs of ONE thread-block cluster fill
    // a run of narrow row-levels in lockstep, one cluster barrier per level)
    constexpr bool DF = DFM == 1;
    constexpr bool CL = DFM == 2;
    constexpr bool RUN = DFM != 0;
// gathers in flight per lane (prefix batch).  The pivot blocks (D13) of the
// u8 shapes are short (M2s: 3-5 prefixes), so a padded batch computes windows
// for empty slots; measured round 2 (solve ms, against 16 / 10): uint8 CH = 1
// 8 and CH = 2 (prefix list in shared memory) 4: M2s 2.24 -> 2.13, M4s 22.6 ->
// 21.7, M4x unchanged; uint16 CH = 2 4 (M3s 7.18 -> 6.88, M3g 47.1 -> 44.9);
// uint16 CH = 1 stays 16 (M3s, 8 was +3 %).  CH = 2 with
// the prefix list in shared memory once took 10 (20 prefixes in two batches:
// M2s -5 % in round 1, before the pivot blocks).
#ifndef PTAS_PB1
#define PTAS_PB1 8
#endif
#ifndef PTAS_PB1U16
#define PTAS_PB1U16 16
#endif
#ifndef PTAS_PB2
#define PTAS_PB2 8
#endif
#ifndef PTAS_PB2S
#define PTAS_PB2S 4
#endif
#ifndef PTAS_PB2U16
#define PTAS_PB2U16 4
#endif
    constexpr int PB = CH == 1 ? (EB == 2 ? PTAS_PB1U16 : PTAS_PB1)
                               : (CH == 2 ? (EB == 2 ? PTAS_PB2U16 : (CPREF ? PTAS_PB2 : PTAS_PB2S)) : 4);
    constexpr bool PB_POW2 = (PB & (PB - 1)) == 0;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    // Programmatic dependent launch: let the next row-level's grid start its
    // prologue now; everything before griddepcontrol.wait below reads only data
    // produced before the first fill launch of the DP (prefix table, row index).
    asm volatile("griddepcontrol.launch_dependents;");
    // enumeration without a host round trip overflowed its bounds (grid-uniform):
    // nothing is filled and the host redoes the DP synchronously
    if (meta->ovf) return;
    const ConstPref &cp = c_pref[CPREF ? cslot : 0];
    const int np = CPREF ? cp.np : (int)(meta->nP - 1);
    // s_oj[c] = oj_entry: int32 offsets (the host routes tables of 2^31 words
    // or more to the scalar kernel); s_w: packed digits
    const int npad = (np + 31) & ~31;  // zero-padded: dummy slots are never loaded (mask bit 0)
    int2 *s_oj = reinterpret_cast<int2 *>(smem_raw);
    // (16 dummy entries past npad: a batch of a non-power-of-two size may run
    // past the last chunk; those slots are never loaded, their mask bit is 0)
    uint64_t *s_w = reinterpret_cast<uint64_t *>(s_oj + npad + 16);
    for (int i = threadIdx.x; i < npad + 16; i += blockDim.x) {
        if (i < np) {
            const PrefixEntry pe = gpref[1 + i];
            if (!CPREF) s_oj[i] = oj_entry(pe, EB);
#pragma unroll
            for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = pe.w[w];
        } else if (!CPREF) {
            s_oj[i] = make_int2(0, (EB == 1 ? SEL_U8 : SEL_U16) + SEL_SELF);
        }
    }
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int rpw = 32 / Lg;
    const int grp = lane / Lg;          // grp >= rpw: idle lane
    const int xl = lane - grp * Lg;
    // nsplit == 1: every warp owns its own rows.  nsplit > 1 (small row-levels):
    // the nsplit warps of a block share one set of rows, each walks every
    // nsplit-th 32-prefix chunk (long prefix lists) or every nsplit-th batch of
    // PB prefixes within each chunk (short lists), and warp 0 combines the partial minima (shared
    // memory) before the chain.
    const int nsplit = SPLIT ? nsplit_arg : 1;
    const int wid = threadIdx.x >> 5;
    const int64_t gw = SPLIT ? (int64_t)blockIdx.x : ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = SPLIT ? (int64_t)gridDim.x : ((int64_t)gridDim.x * blockDim.x) >> 5;
    const bool split_chunks = SPLIT && np >= 32 * nsplit;
    const int pbase0 = split_chunks ? wid * 32 : 0;
    const int pstep = split_chunks ? nsplit * 32 : 32;
    const int qbase0 = (SPLIT && !split_chunks) ? wid * PB : 0;
    const int qstep = (SPLIT && !split_chunks) ? nsplit * PB : PB;
    uint32_t *s_red = reinterpret_cast<uint32_t *>(s_w + (size_t)NW * np + 1);  // [warp][2][CH][32]
    uint64_t guard[NW], maxs[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        guard[w] = g.guard[w];
        maxs[w] = g.maxs[w];
    }
    // DF: per-level first set / first slot of the run, in shared memory
    int32_t *s_set = reinterpret_cast<int32_t *>(s_red + (size_t)(256 / 32) * 2 * CH * 32);
    int32_t *s_sl = s_set + (RUN ? df.nlev + 1 : 0);
    // DF + SPLIT: the block's ticket (8-byte aligned after the plan)
    unsigned long long *s_tk =
        reinterpret_cast<unsigned long long *>(s_set + ((RUN ? 2 * (df.nlev + 1) : 0) + 1) / 2 * 2);
    // dominance table (g.TS > 0, D10): per-digit selectors, then the
    // chunk words (copied from the DP's table built after the prefix list)
    // (offset arithmetic from smem_raw keeps the shared state space: LDS, not generic loads)
    // pivot blocks (D13) and the packed-bit -> leading-digit map
    int32_t *s_blk = reinterpret_cast<int32_t *>(s_tk + 1);
    int8_t *s_b2d = reinterpret_cast<int8_t *>(s_blk + 2 * MAXK);
    int4 *s_dsel = reinterpret_cast<int4 *>(
        smem_raw + ((reinterpret_cast<unsigned char *>(s_b2d + NW * 64) - smem_raw + 15) & ~(ptrdiff_t)15));
    uint32_t *s_tab = reinterpret_cast<uint32_t *>(s_dsel + g.K1);
    // (uint8 kernels only: in the 64-register uint16 kernels the extra code
    // costs more than it saves, measured)
    const bool use_tab = EB == 1 && g.TS > 0;
    if (EB == 1 && use_tab) {
        for (int i = threadIdx.x; i < g.K1; i += blockDim.x) {
            const uint64_t gw = g.guard[g.word[i]] >> g.shift[i];
            s_dsel[i] = make_int4(g.shift[i] | (g.word[i] << 8), (int)((gw & (~gw + 1)) - 1), g.hi[i], g.dbase[i]);
        }
        const int n = ((np + 31) >> 5) * g.TS;
        for (int e = threadIdx.x; e < n; e += blockDim.x) s_tab[e] = g.domtab[e];
        __syncthreads();
    }
    for (int i = threadIdx.x; i < 2 * MAXK + NW * 64; i += blockDim.x) {
        if (i < 2 * MAXK) {
            s_blk[i] = i < 2 * g.K1 ? g.blk[i] : 0;
        } else {
            const int b = i - 2 * MAXK, wd = b >> 6, bit = b & 63;
            int d = -1;
            for (int q = 0; q < g.K1; ++q)
                if (g.word[q] == wd && g.shift[q] <= bit) d = q;
            s_b2d[b] = (int8_t)d;
        }
    }
    if constexpr (RUN) {
        for (int i = threadIdx.x; i < 2 * (df.nlev + 1); i += blockDim.x) s_set[i] = df.plan[i];
    }
    __syncthreads();
    // first row set's index entries, loaded before waiting on the previous level
    int64_t nrb = 0;
    uint64_t npw[NW];
    // CL: warp gwc of the cluster takes sets gwc, gwc + nwc, ... of each level
    int c_lv = 0, n_lv = 0, bars = 0;
    int64_t c_t = 0, n_t = 0;
    int gwc = 0, nwc = 1;
    auto cl_norm = [&](int &lv, int64_t &t) {
        while (lv < df.nlev && t >= (int64_t)(s_set[lv + 1] - s_set[lv])) {
            ++lv;
            t = gwc;
        }
    };
    auto cl_load = [&](int lv, int64_t t) {
        const int64_t sl = (int64_t)s_sl[lv] + t * rpw + grp;
        const bool ok = grp < rpw && sl < s_sl[lv + 1];
#pragma unroll
        for (int w = 0; w < NW; ++w) npw[w] = ok ? pwa[(int64_t)w * pw_stride + sl] : 0;
        nrb = ok ? rb[sl] : 0;
    };
    if constexpr (CL) {
        uint32_t r, nr;
        asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
        asm("mov.u32 %0, %%cluster_nctarank;" : "=r"(nr));
        gwc = (int)r * (int)(blockDim.x >> 5) + wid;
        nwc = (int)nr * (int)(blockDim.x >> 5);
        c_t = gwc;
        cl_norm(c_lv, c_t);
        if (c_lv < df.nlev) cl_load(c_lv, c_t);
    } else if constexpr (!DF) {
        const int64_t slot = gw * rpw + grp;
        const bool ok = grp < rpw && slot < slot_count;
#pragma unroll
        for (int w = 0; w < NW; ++w) npw[w] = ok ? pwa[(int64_t)w * pw_stride + slot_begin + slot] : 0;
        if (ok) nrb = rb[slot_begin + slot];
    }
    asm volatile("griddepcontrol.wait;" ::: "memory");

    // DF row sets: tickets in level order; set t of level lv covers slots
    // s_sl[lv] + (t - s_set[lv]) * rpw + grp (< s_sl[lv+1])
    int df_lv = 0;            // level (within the run) of the last mapped ticket
    int64_t tk = 0;          // current ticket
    int cur_lv = 0;
    int64_t cur_slot = 0, nxt_slot = 0;
    bool cur_ok = false, nxt_ok = false;
    const uint32_t Lw = (uint32_t)(g.Wp * EB / 4);
    auto df_map = [&](int64_t t, int64_t &slot, bool &ok) {
        while (t >= s_set[df_lv + 1]) ++df_lv;
        slot = (int64_t)s_sl[df_lv] + (t - s_set[df_lv]) * rpw + grp;
        ok = grp < rpw && slot < s_sl[df_lv + 1];
    };
    if constexpr (DF) {
        unsigned long long t0 = 0;
        if (SPLIT) {
            if (threadIdx.x == 0) *s_tk = atomicAdd(df.ticket, 1ull);
            __syncthreads();
            t0 = *s_tk;
            __syncthreads();   // every warp has read it before thread 0 stores the next ticket
        } else {
            if (lane == 0) t0 = atomicAdd(df.ticket, 1ull);
            t0 = __shfl_sync(FULL, t0, 0);
        }
        tk = (int64_t)(t0 - df.base);
        if (tk < df.total_sets) {
            df_map(tk, cur_slot, cur_ok);
            cur_lv = df_lv;
#pragma unroll
            for (int w = 0; w < NW; ++w) npw[w] = cur_ok ? pwa[(int64_t)w * pw_stride + cur_slot] : 0;
            if (cur_ok) nrb = rb[cur_slot];
        }
    }

    const uint32_t *tab32 = reinterpret_cast<const uint32_t *>(table);
    // uniform trip count (every warp of the grid runs the same number of row
    // sets; the tail ones are idle) keeps the prefix loop in uniform control flow
    const int64_t nsets = (slot_count + rpw - 1) / rpw;
    const int64_t iters = RUN ? 0 : (nsets + nw - 1) / nw;
    for (int64_t it = 0;; ++it) {
        if (CL ? c_lv >= df.nlev : (DF ? tk >= df.total_sets : it >= iters)) break;
        const int64_t sb = (it * nw + gw) * rpw;
        const int64_t slot = CL ? (int64_t)s_sl[c_lv] + c_t * rpw + grp : (DF ? cur_slot : sb + grp);
        const bool rowok = CL ? (grp < rpw && slot < s_sl[CL ? c_lv + 1 : 0]) : (DF ? cur_ok : (grp < rpw && slot < slot_count));
        const int64_t rowbase = nrb;
        uint64_t pw[NW];
        bool row0 = rowok;   // p = 0 (all leading digits zero)
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            pw[w] = npw[w] | (rowok ? g.pw_or[w] : 0ull);
            row0 &= pw[w] == 0;
        }
        unsigned long long tnext = 0;
        if constexpr (CL) {
            // next set of this warp (possibly levels ahead) and its index entries
            n_lv = c_lv;
            n_t = c_t + nwc;
            cl_norm(n_lv, n_t);
            if (n_lv < df.nlev) cl_load(n_lv, n_t);
            // every level below c_lv is complete in the whole cluster
            // (release/acquire at cluster scope orders the table stores)
            while (bars < c_lv) {
                asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
                ++bars;
            }
        } else if constexpr (DF) {
            // next ticket now; its value is consumed after the prefix walk
            if (SPLIT ? threadIdx.x == 0 : lane == 0) tnext = atomicAdd(df.ticket, 1ull);
        } else {   // prefetch the next row set's index entries
            const int64_t ns = sb + nw * rpw + grp;
            const bool ok = grp < rpw && ns < slot_count;
#pragma unroll
            for (int w = 0; w < NW; ++w) npw[w] = ok ? pwa[(int64_t)w * pw_stride + slot_begin + ns] : 0;
            nrb = ok ? rb[slot_begin + ns] : 0;
        }
        // the lane's first word (int32 word index: the launcher guarantees < 2^31 words)
        const uint32_t *src = tab32 + ((int)(rowbase * EB / 4) + xl * CH);
        // opaque to the compiler: keeps the pointer in registers instead of
        // re-deriving it from the kernel parameters at every gather
        asm volatile("" : "+l"(src));
        uint32_t rid = 0;   // DF: row-major row id of the group's row (flag index)
#if PTAS_DF_PROFILE
        long long pf_t0 = clock64(), pf_t1 = 0, pf_t2 = 0;
#endif
        if constexpr (DF) {
            rid = rowok ? (uint32_t)(rowbase * EB / 4) / Lw : 0u;
            if (cur_lv > 0) {
                uint32_t sleep_ns = (uint32_t)df.sleep0;
                // wait until every unit predecessor p - e_i (p_i >= 1) is done; by
                // induction that covers every dominated row, i.e. every source
                // row p - s' of the prefix walk (rows of the run's first level
                // read only rows filled before the launch)
                for (;;) {
                    bool ok = true;
                    if (rowok) {
                        for (int i = xl; i < g.K1; i += Lg) {
                            const uint64_t wv = NW == 1 ? pw[0] : (g.word[i] ? pw[NW - 1] : pw[0]);
                            if (wv & df.dmask[i]) {
                                const uint32_t *f = df.flags + (rid - (uint32_t)df.rstride[i]);
#if PTAS_DF_NOACQ   // measurement only (not a correct protocol): flags without acquire
                                uint32_t fv;
                                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(fv) : "l"(f) : "memory");
                                ok &= fv == df.epoch;
#else
                                ok &= ld_acquire(f) == df.epoch;
#endif
                            }
                        }
                    }
                    if (__all_sync(FULL, ok)) break;
                    __nanosleep(sleep_ns);
                    if (sleep_ns < df.sleep_max) sleep_ns *= 2;   // backoff (fewer polls, fewer L1 invalidations)
                }
                __syncwarp();
            }
        }
        // every prefix dominated by every row of the warp?
        bool interior = rowok;
#pragma unroll
        for (int w = 0; w < NW; ++w) interior &= (((pw[w] | guard[w]) - maxs[w]) & guard[w]) == guard[w];
        const bool allint = __all_sync(FULL, grp >= rpw || interior);

#if PTAS_DF_PROFILE
        pf_t1 = clock64();
        unsigned long long pf_g1 = 0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(pf_g1));
#endif
        // ---- pivot block of the row (D13): prefixes whose first nonzero digit is
        // the row's first nonzero digit; row 0 and idle lanes: empty
        int plo = 0, phi = 0;
        if (rowok) {
            const int b0 = NW == 1 || pw[0] ? __ffsll((long long)pw[0]) - 1 : (NW > 1 && pw[NW - 1] ? 63 + __ffsll((long long)pw[NW - 1]) : -1);
            if (b0 >= 0) {
                const int q = s_b2d[b0];
                plo = s_blk[2 * q];
                phi = s_blk[2 * q + 1];
            }
        }
        const int wlo = __reduce_min_sync(FULL, plo < phi ? plo : INT32_MAX);
        const int whi = __reduce_max_sync(FULL, phi);
        // ---- cross-row relaxations: acc = min over s' <= p in the block of OPT(p - s', x - min(x, Jmax(s')))
        Words<CH> ae, ao;
        fill_words(ae, 0xffffffffu);
        fill_words(ao, 0xffffffffu);
        for (int base = (whi > 0 ? (wlo & ~31) : np) + pbase0; base < whi; base += pstep) {
            const int cnt = whi - base < 32 ? whi - base : 32;
            // the row's block within this chunk
            const int rl = min(max(plo - base, 0), 32), rh = min(max(phi - base, 0), 32);
            const unsigned rmask = (rh >= 32 ? FULL : ((1u << rh) - 1u)) & ~(rl >= 32 ? FULL : ((1u << rl) - 1u));
            unsigned m;
            if (allint) {
                m = !rowok ? 0u : rmask;  // idle lanes load nothing
            } else {
                // lane xl tests prefixes base + xl + k*Lg for its group's row (uniform
                // trip count), then an OR all-reduce over the group by rotations
                // (after the step with distance d every lane holds the OR of 2d
                // consecutive group lanes; OR is idempotent, so overlaps are harmless)
                unsigned bits = 0;
                if (EB == 1 && use_tab) {
                    // AND over the row's digits of the chunk's table words, the digits
                    // spread over the group's lanes, then an AND all-reduce over the group
                    bits = 0xffffffffu;
                    const uint32_t *tb = s_tab + (base >> 5) * g.TS;
                    for (int i = xl; i < g.K1; i += Lg) {
                        const int4 d = s_dsel[i];
                        const uint64_t wv = NW == 1 ? pw[0] : ((d.x >> 8) ? pw[NW - 1] : pw[0]);
                        const int v = min((int)((uint32_t)(wv >> (d.x & 0xff)) & (uint32_t)d.y), d.z);
                        bits &= tb[d.w + v];
                    }
                    for (int d = 1; d < Lg; d <<= 1) {
                        const int xs = xl + d >= Lg ? xl + d - Lg : xl + d;
                        bits &= __shfl_sync(FULL, bits, lane - xl + xs);
                    }
                    bits &= cnt == 32 ? FULL : ((1u << cnt) - 1u);
                }
                for (int c0 = 0; c0 < (use_tab ? 0 : cnt); c0 += Lg) {   // ceil(cnt / Lg) steps, no division
                    const int c = xl + c0;
                    const bool in = rowok && c < cnt;
                    const int ci = base + (in ? c : 0);
                    bool dom = in;
#pragma unroll
                    for (int w = 0; w < NW; ++w)
                        dom &= (((pw[w] | guard[w]) - s_w[(size_t)w * np + ci]) & guard[w]) == guard[w];
                    bits |= dom ? (1u << c) : 0u;
                }
                for (int d = 1; d < (use_tab ? 1 : Lg); d <<= 1) {
                    const int xs = xl + d >= Lg ? xl + d - Lg : xl + d;
                    bits |= __shfl_sync(FULL, bits, lane - xl + xs);
                }
                m = rowok ? bits & rmask : 0u;  // idle lanes (past 32 / Lg groups) may have read foreign bits
            }
            const int cend = PB_POW2 ? ((cnt + PB - 1) & ~(PB - 1)) : (cnt + PB - 1) / PB * PB;
            // first batch holding a prefix of the warp's blocks (the chunk may start below them)
            const int qlo = wlo > base ? (PB_POW2 ? ((wlo - base) & ~(PB - 1)) : (wlo - base) / PB * PB) : 0;
            // PB prefixes per step: their gathers are issued before any is consumed
            for (int q0 = qlo + qbase0; q0 < cend; q0 += qstep) {
                Words<CH> cur[PB];
                int sj[PB];
#pragma unroll
                for (int u = 0; u < PB; ++u) {
                    const int q = q0 + u;
                    const int2 oj = CPREF ? cp.oj[base + q] : s_oj[base + q];
                    sj[u] = oj.y;
                    const uint32_t *p = src + oj.x;
                    if (PB_POW2 ? ((m >> q) & 1u) : (q < 32 && ((m >> (q & 31)) & 1u))) cur[u] = load_words<CH, RUN>(p);
                    else fill_words(cur[u], 0xffffffffu);
                }
#pragma unroll
                for (int u = 0; u < PB; ++u) {
                    const uint32_t sel = (uint32_t)sj[u];   // warp-uniform
                    Words<CH> lo, hi;
                    // positions before the row read its first entry (clamp to x = 0)
                    // (db <= 4: only lane xl = 0 reads it, from its own word 0).
                    // Jmax(s') = 0 needs no window: its selector reads `hi` only.
                    uint32_t f = cur[u].v[0];
                    if (WIN != 4 && (sel >> 16) > 4u) f = __shfl_sync(FULL, f, lane - xl);
                    f = EB == 1 ? prmt(f, 0u, 0x0000u) : prmt(f, 0u, 0x1010u);
                    windows<CH, WIN>(cur[u], (int)(sel >> 16), xl, f, lo, hi);
#pragma unroll
                    for (int t = 0; t < CH; ++t) {
                        if constexpr (EB == 1) {
                            ae.v[t] = vmin2(ae.v[t], prmt(lo.v[t], hi.v[t], sel));
                            ao.v[t] = vmin2(ao.v[t], prmt(lo.v[t], hi.v[t], sel + 0x1111u));
                        } else {
                            ae.v[t] = vmin2(ae.v[t], prmt(lo.v[t], hi.v[t], sel));
                        }
                    }
                }
            }
        }

        // DF: next row set -- map the ticket and start its index loads (they
        // land during the in-row closure)
        auto df_next = [&](unsigned long long t) {
            const int64_t tn = (int64_t)(t - df.base);
            nxt_ok = false;
            if (tn < df.total_sets) df_map(tn, nxt_slot, nxt_ok);
#pragma unroll
            for (int w = 0; w < NW; ++w) npw[w] = nxt_ok ? pwa[(int64_t)w * pw_stride + nxt_slot] : 0;
            nrb = nxt_ok ? rb[nxt_slot] : 0;
            tk = tn;
        };
#if PTAS_DF_PROFILE
        pf_t2 = clock64();
#endif
        if constexpr (DF && !SPLIT) df_next(__shfl_sync(FULL, tnext, 0));
        if (SPLIT) {
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                s_red[((wid * 2 + 0) * CH + t) * 32 + lane] = ae.v[t];
                s_red[((wid * 2 + 1) * CH + t) * 32 + lane] = ao.v[t];
            }
            if (DF && threadIdx.x == 0) *s_tk = tnext;
            __syncthreads();
            if constexpr (DF) df_next(*s_tk);
            if (wid == 0) {
                for (int w2 = 1; w2 < nsplit; ++w2) {
#pragma unroll
                    for (int t = 0; t < CH; ++t) {
                        ae.v[t] = vmin2(ae.v[t], s_red[((w2 * 2 + 0) * CH + t) * 32 + lane]);
                        ao.v[t] = vmin2(ao.v[t], s_red[((w2 * 2 + 1) * CH + t) * 32 + lane]);
                    }
                }
            }
        }
        if (!SPLIT || wid == 0) {
            // ---- OPT(p, x) = 1 + acc(x) for p != 0 (D12); row p = 0: ceil(x / J0)
            // uint8: E holds x = 4w, 4w+2; O holds x = 4w+1, 4w+3 (uint16 lanes).
            // uint16: E holds 2w, 2w+1.  Every row p != 0 dominates a unit prefix of
            // its pivot block, so acc is finite there.
            Words<CH> oe, oo;
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                if constexpr (EB == 1) {
                    oe.v[t] = (ae.v[t] & 0x00ff00ffu) + ONES;
                    oo.v[t] = (ao.v[t] & 0x00ff00ffu) + ONES;
                } else {
                    oe.v[t] = vmin2(ae.v[t], 0xfffefffeu) + ONES;
                    oo.v[t] = 0;
                }
            }
            if (row0) {   // row p = 0 (once per DP): OPT(0, x) = ceil(x / J0)
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    const uint32_t x0 = (uint32_t)(xl * CH + t) * (4 / EB);
                    auto cf = [&](uint32_t x) { return (x + (uint32_t)J0 - 1u) / (uint32_t)J0; };
                    if constexpr (EB == 1) {
                        oe.v[t] = cf(x0) | (cf(x0 + 2) << 16);
                        oo.v[t] = cf(x0 + 1) | (cf(x0 + 3) << 16);
                    } else {
                        oe.v[t] = cf(x0) | (cf(x0 + 1) << 16);
                    }
                }
            }
            // ---- store the packed row (padding bytes receive don't-care values)
            if (rowok) {
                uint32_t *out32 = compact ? reinterpret_cast<uint32_t *>(compact + slot * g.Wp)
                                          : reinterpret_cast<uint32_t *>(table + rowbase);
                Words<CH> wv;
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    if constexpr (EB == 1) wv.v[t] = prmt(oe.v[t], oo.v[t], 0x6240u);
                    else wv.v[t] = oe.v[t];
                }
                store_words<CH>(out32 + xl * CH, wv);
            }
            if constexpr (DF) {
                // release: the row's words are visible at gpu scope before its flag
                __threadfence();
                __syncwarp();
                if (rowok && xl == 0) st_relaxed(df.flags + rid, df.epoch);
#if PTAS_DF_PROFILE
                // per level (of the run): sets, wait, walk, tail cycles, first ready, last done (ns)
                if (df.prof && lane == 0) {
                    unsigned long long g2;
                    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g2));
                    unsigned long long *pr = df.prof + 6 * (size_t)cur_lv;
                    atomicAdd(pr + 0, 1ull);
                    atomicAdd(pr + 1, (unsigned long long)(pf_t1 - pf_t0));
                    atomicAdd(pr + 2, (unsigned long long)(pf_t2 - pf_t1));
                    atomicAdd(pr + 3, (unsigned long long)(clock64() - pf_t2));
                    atomicMin(pr + 4, pf_g1);
                    atomicMax(pr + 5, g2);
                }
#endif
            }
            __syncwarp();
        }  // chain + store (warp 0 in split mode)
        if (SPLIT) __syncthreads();  // s_red reused by the next row set
        if constexpr (DF) {
            cur_slot = nxt_slot;
            cur_ok = nxt_ok;
            cur_lv = df_lv;
        }
        if constexpr (CL) {
            c_lv = n_lv;
            c_t = n_t;
        }
    }
    if constexpr (CL) {
        // every thread of the cluster passes the same nlev - 1 barriers
        while (bars < df.nlev - 1) {
            asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
            ++bars;
        }
    }
}

// Resident blocks per SM of a kernel variant at a dynamic smem size (cached).
template <typename K>
static int occupancy_of(K kfn, size_t smem, int bs)
{
    static std::mutex mu;
    static std::unordered_map<uint64_t, int> cache;
    const uint64_t key = (uint64_t)(uintptr_t)(const void *)kfn ^ ((uint64_t)smem << 40);
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kfn, bs, smem) != cudaSuccess || occ < 1) occ = 1;
    cache[key] = occ;
    return occ;
}

// Words per lane CH for a row of Lw words (group width Lg = Lw / CH <= 32),
// 0 = the packed kernel does not support the geometry.  CH amortises the
// per-prefix cost over CH words; small row-levels are latency-bound and use
// CH = 1 (more lanes per row, shorter serial work per lane).  `rows` = rows
// of the level (per-level launches) or of the largest level of the run (DF).
static int plan_ch(int e, const RowGeom &g, int J0, int64_t rows, int sm_count, bool df)
{
    const int Lw = (int)(g.Wp * e / 4);
    if ((g.Wp * e) % 4 != 0 || Lw > 256 || J0 * e > 124) return 0;
    // int32 word offsets: the table (incl. padding) must stay below 2^31 words
    int64_t rows_all = 1;
    for (int i = 0; i < g.K1; ++i) rows_all *= (int64_t)g.N[i] + 1;
    if ((g.span_words > 0 ? g.span_words : rows_all * (int64_t)Lw) >= ((int64_t)1 << 31)) return 0;
    int CH;
    const int64_t chs = df ? PTAS_KNOB("PTAS_DF_CH", 0) : PTAS_KNOB("PTAS_SWAR_CH", 0);
    const int64_t cht = PTAS_KNOB("PTAS_SMALL_LEVEL_ROWS", -1);
    const int64_t small_rows = cht >= 0 ? cht : (int64_t)sm_count * 32;
    if (Lw > 32) CH = Lw <= 64 ? 2 : (Lw <= 128 ? 4 : 8);
    else if (chs > 0) CH = (int)chs;
    else CH = (Lw >= 8 && rows > small_rows) ? 2 : 1;
    if (CH != 1 && CH != 2 && CH != 4 && CH != 8) CH = 1;
    if (Lw % CH != 0) {
        if (Lw > 32) return 0;
        CH = 1;
    }
    const int Lg = Lw / CH;
    if (Lg < 1 || Lg > 32) return 0;
    return CH;
}

static size_t swar_smem(int64_t np, int NW, int nlev_df, const RowGeom &g, int CH)
{
    // s_oj | s_w | pad | s_red | DF plan | ticket (16 B) | dominance selectors + table
    // (s_red sized for the kernel's lane chunk: smem left over is L1 for the gathers)
    return (size_t)((np + 31) & ~31) * 8 + 16 * 8 + (size_t)np * 8 * NW + 16 + (size_t)(256 / 32) * 2 * CH * 32 * 4 +
           (size_t)8 * (nlev_df + 1) + 32 + (size_t)8 * MAXK + (size_t)64 * NW + 16 +
           (g.TS > 0 ? (size_t)16 * g.K1 + (size_t)((np + 31) / 32) * g.TS * 4 : 0);
}

// Host launcher body for one (E, NW): returns cudaErrorNotSupported when the
// geometry needs the scalar kernel (row longer than 1 KiB, pitch not a
// multiple of the lane chunk, or a table of 2^31 words or more).
// df != nullptr: one dataflow launch over the run described by *df.
template <typename E, int NW>
static cudaError_t launch_swar_impl(int e, void *table, const RowGeom &g, const int64_t *rb,
                                 const uint64_t *pw, int64_t pw_stride, const PrefixEntry *d_pref,
                                 const DpMeta *d_meta, int64_t nP_bound, int J0, int rho,
                                 int64_t slot_begin, int64_t slot_count, void *compact_out, int sm_count,
                                 cudaStream_t st, int pdl, int cslot, const DfArgs *df = nullptr,
                                 unsigned long long *ticket_base = nullptr)
{
    if (slot_count <= 0) return cudaSuccess;
    if (compact_out && ((uintptr_t)compact_out & 15)) return cudaErrorNotSupported;
    const int CH = plan_ch(e, g, J0, slot_count, sm_count, df != nullptr);
    if (CH == 0) return cudaErrorNotSupported;
    const int Lw = (int)(g.Wp * e / 4);
    const int Lg = Lw / CH;
    const int rpw = 32 / Lg;
    const int bs = 256;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;   // bound: sizes the shared-memory tables
    // heuristics use the caller's estimate when the exact length is not known on the host
    const int64_t nph = tl_np_hint >= 0 ? std::min<int64_t>(tl_np_hint, np) : np;
    // small row-levels with long prefix lists: split each row set's prefixes over the 8 warps of a block
    const int64_t sp = PTAS_KNOB("PTAS_SPLIT_ROWS", -1);
    // (worth it when a row's prefix walk has several batches of gathers in series)
    const int PBh = CH == 1 ? (e == 2 ? PTAS_PB1U16 : PTAS_PB1) : (CH == 2 ? PTAS_PB2 : 4);
    const int64_t split_rows = sp >= 0 ? sp : ((nph + PBh - 1) / PBh >= 4 ? (int64_t)sm_count * rpw * 2 : 0);
    // df->nsplit: 1 = warp row sets, 8 = block row sets, 0 = one cluster in lockstep
    const bool cl = df && df->nsplit == 0;
    const int64_t cls = PTAS_KNOB("PTAS_CL_SIZE", 16);
    const int cl_size = cl ? (int)std::max<int64_t>(1, std::min<int64_t>(16, cls)) : 1;
    const int nsplit = df ? (df->nsplit > 1 ? bs / 32 : 1) : (slot_count <= split_rows ? bs / 32 : 1);
    const size_t smem = swar_smem(np, NW, df ? df->nlev : 0, g, CH);
    if (smem > 220 * 1024) return cudaErrorNotSupported;
    // shifts beyond one word: prefix windows J * e (J <= J0) or chain u16-lane shifts
    // prefix windows beyond two words (J * e > 8, J <= J0) need the generic word fetch;
    // the in-row closure handles any shift (registers up to 8 bytes, else shared memory)
    const int win = J0 * e <= 4 ? 4 : (J0 * e <= 8 ? 8 : 0);
    const bool cpref = np <= CP_MAX && cslot >= 0 && cslot < CP_SLOTS && nph >= 64;
    const int64_t df_wave = std::max<int64_t>(1, PTAS_KNOB("PTAS_DF_WAVE", 2));
    DfArgs dfa;
    if (df) dfa = *df;
    else std::memset(&dfa, 0, sizeof(dfa));
    cudaError_t err;
#define PTAS_SWAR_GO(E_, NW_, CH_, WIN_)                                                                  \
    do {                                                                                                  \
        auto kfn = cl ? (cpref ? row_fill_swar_kernel<E_, NW_, CH_, WIN_, true, false, 2>                 \
                               : row_fill_swar_kernel<E_, NW_, CH_, WIN_, false, false, 2>)               \
                 : df ? (cpref ? (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, WIN_, true, true, 1>    \
                                             : row_fill_swar_kernel<E_, NW_, CH_, WIN_, true, false, 1>)  \
                               : (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, WIN_, false, true, 1>   \
                                             : row_fill_swar_kernel<E_, NW_, CH_, WIN_, false, false, 1>)) \
               : cpref ? (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, WIN_, true, true, 0>            \
                                     : row_fill_swar_kernel<E_, NW_, CH_, WIN_, true, false, 0>)          \
                       : (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, WIN_, false, true, 0>           \
                                     : row_fill_swar_kernel<E_, NW_, CH_, WIN_, false, false, 0>);        \
        if (smem > 48 * 1024) {                                                                           \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);      \
            if (err != cudaSuccess) return err;                                                           \
        }                                                                                                 \
        {   /* PTAS_CARVEOUT=<pct> (experiment): preferred shared-memory carveout */                     \
            static const int co = [] { const char *t = std::getenv("PTAS_CARVEOUT");                     \
                                       return t && t[0] ? std::atoi(t) : -1; }();                          \
            if (co >= 0) cudaFuncSetAttribute(kfn, cudaFuncAttributePreferredSharedMemoryCarveout, co);    \
        }                                                                                                 \
        if (cl && cl_size > 8) {                                                                          \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);           \
            if (err != cudaSuccess) return err;                                                           \
        }                                                                                                 \
        int64_t blocks;                                                                                   \
        const int64_t cap = (int64_t)sm_count * occupancy_of(kfn, smem, bs);                              \
        if (cl) {                                                                                         \
            blocks = cl_size;   /* one cluster */                                                         \
        } else if (df) {                                                                                  \
            /* persistent: every block resident, row sets from the ticket counter */                     \
            const int spb = nsplit > 1 ? 1 : bs / 32;   /* row sets in flight per block */                \
            /* enough row sets in flight for `wave` of the run's widest levels: more would only spin */   \
            const int64_t inflight = std::min<int64_t>(df->total_sets, df_wave * ((slot_count + rpw - 1) / rpw)); \
            blocks = (inflight + spb - 1) / spb;                                                          \
            const int64_t capd = df->grid_div > 1 ? std::max<int64_t>(1, cap / df->grid_div) : cap;      \
            if (blocks > capd) blocks = capd;                                                             \
        } else if (nsplit > 1) {                                                                          \
            blocks = (slot_count + rpw - 1) / rpw;                                                        \
        } else {                                                                                          \
            /* one resident wave: every warp loops over row sets */                                       \
            blocks = (slot_count + (int64_t)(bs / 32) * rpw - 1) / ((int64_t)(bs / 32) * rpw);           \
            if (blocks > cap) blocks = cap;                                                               \
        }                                                                                                 \
        cudaLaunchConfig_t cfg = {};                                                                      \
        cudaLaunchAttribute attr[2];                                                                      \
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;                                  \
        attr[0].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;                                 \
        attr[1].id = cudaLaunchAttributeClusterDimension;                                                 \
        attr[1].val.clusterDim.x = (unsigned)cl_size;                                                     \
        attr[1].val.clusterDim.y = 1;                                                                     \
        attr[1].val.clusterDim.z = 1;                                                                     \
        cfg.gridDim = dim3((unsigned)blocks);                                                             \
        cfg.blockDim = dim3(bs);                                                                          \
        cfg.dynamicSmemBytes = smem;                                                                      \
        cfg.stream = st;                                                                                  \
        cfg.attrs = attr;                                                                                 \
        cfg.numAttrs = cl ? 2 : 1;                                                                        \
        err = cudaLaunchKernelEx(&cfg, kfn, (E_ *)table, g, rb, pw, pw_stride, d_pref, d_meta, J0, rho,   \
                                 slot_begin, slot_count, (E_ *)compact_out, Lg, nsplit, cslot, dfa);      \
        if (err != cudaSuccess) return err;                                                               \
        /* every grabbing warp (block in split mode) ends with exactly one failed grab */               \
        if (df && !cl && ticket_base) *ticket_base += (unsigned long long)df->total_sets +                \
                                                      (unsigned long long)blocks * (nsplit > 1 ? 1 : bs / 32); \
    } while (0)
#define PTAS_SWAR_CASE(E_, NW_, CH_)                                                              \
    do {                                                                                          \
        if (win == 4) PTAS_SWAR_GO(E_, NW_, CH_, 4);                                              \
        else if (win == 8) PTAS_SWAR_GO(E_, NW_, CH_, 8);                                         \
        else PTAS_SWAR_GO(E_, NW_, CH_, 0);                                                       \
    } while (0)
    if (CH == 1) PTAS_SWAR_CASE(E, NW, 1);
    else if (CH == 2) PTAS_SWAR_CASE(E, NW, 2);
    else if (CH == 4) PTAS_SWAR_CASE(E, NW, 4);
    else PTAS_SWAR_CASE(E, NW, 8);
#undef PTAS_SWAR_CASE
#undef PTAS_SWAR_GO
    return cudaGetLastError();
}

template <typename E, int NW>
static cudaError_t launch_swar_df_impl(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                       int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                       int64_t nP_bound, int J0, int64_t max_level_rows, const DfArgs &df,
                                       unsigned long long *ticket_base, int sm_count, cudaStream_t st, int pdl,
                                       int cslot)
{
    if (df.total_sets <= 0) return cudaSuccess;
    return launch_swar_impl<E, NW>(e, table, g, rb, pw, pw_stride, d_pref, d_meta, nP_bound, J0, 0, 0,
                                   max_level_rows, nullptr, sm_count, st, pdl, cslot, &df, ticket_base);
}

}  // namespace swar
}  // namespace ptas
