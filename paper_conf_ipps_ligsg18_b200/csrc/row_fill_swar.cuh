// row_fill_swar.cuh — packed-word level fill kernel template (see row_fill_swar.cu).
// Included by the four instantiation units row_fill_swar_<E>_nw<NW>.cu so the
// 48 variants of each (entry type, digit words) pair compile in parallel.
#pragma once
//
// Same recurrence and row-wavefront as row_fill_kernel (dp_kernels.cu), Eq. 1
// of PAPER.md:74-79, but every lane owns one 32-bit word of a row: 4 uint8
// states or 2 uint16 states.  Rows are padded to a multiple of 4 bytes
// (RowGeom::Wp), so every row and every off(s') is word aligned:
//
//   * the source row p - s' of a prefix is read with ONE coalesced 32-bit
//     load per lane;
//   * the j-shifted windows (s = (s', j), j = 0..Jmax(s')) come from the
//     lane's word and its left neighbours (warp shuffles) through one PRMT
//     each; uint8 windows are split into even/odd uint16 lanes with the
//     sign-replicating PRMT mode (v < 128 -> v, v >= 128 -> 0xFF00|v, a
//     monotone encoding), so VIMNMX.U16x2 takes two minima per instruction;
//   * all row groups of a warp walk the prefix list in lockstep (uniform
//     loop, uniform Jmax), each with its own dominance predicate s' <= p.
//
// The in-row term (s' = 0, j = 1..J0) is then resolved on packed uint16
// lanes by Bellman-Ford rounds (shift, +1, min) until no lane changes.
// Every (n, s) with s in C, s <= n is relaxed exactly once, so the closed
// form relaxation count still holds.  Entries in the row padding and in
// lanes past the row end are computed but never read as sources.
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "internal.h"

namespace ptas {
namespace swar {

namespace {

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel)
{
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

__device__ __forceinline__ uint32_t vmin2(uint32_t a, uint32_t b) { return __vminu2(a, b); }

template <int CH>
struct Words {
    uint32_t v[CH];
};

// Lane geometry: a row is owned by a group of Lg lanes (any 1 <= Lg <= 32,
// rows per warp = 32 / Lg, trailing lanes idle); lane xl of group grp holds
// the row's words w = xl + Lg * t, t < CH.
struct LaneMap {
    int lane, Lg, grp, xl;
};

// Word k positions to the left of the lane's word of chunk t.  With
// k = qk * Lg + rk, word w - k lives in lane (xl - rk) mod Lg of the same
// group, chunk t - qk (or t - qk - 1 when the lane index wraps).  Chunks
// before 0 are outside the row and read as `fill`.
template <int CH>
__device__ __forceinline__ uint32_t word_left(const Words<CH> &a, int t, int k, const LaneMap &lm, uint32_t fill)
{
    int qk = 0, rk = k;
    if (k >= lm.Lg) {
        qk = k / lm.Lg;
        rk = k - qk * lm.Lg;
    }
    const int c1 = t - qk, c2 = c1 - 1;
    uint32_t v1 = fill, v2 = fill;
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        if (c == c1) v1 = a.v[c];
        if (c == c2) v2 = a.v[c];
    }
    if (rk == 0) return v1;
    const uint32_t send = (lm.xl >= lm.Lg - rk) ? v2 : v1;
    const int src = lm.lane - rk + (lm.xl < rk ? lm.Lg : 0);
    return __shfl_sync(FULL, send, src);
}

// acc <- min(acc, window of `lo:hi` at byte offset o) for one word position.
template <int EB>
__device__ __forceinline__ void acc_window(uint32_t lo, uint32_t hi, int o, uint32_t &ae, uint32_t &ao)
{
    if constexpr (EB == 1) {
        ae = vmin2(ae, prmt(lo, hi, 0xA280u + 0x1111u * o));
        ao = vmin2(ao, prmt(lo, hi, 0xB391u + 0x1111u * o));
    } else {
        ae = vmin2(ae, prmt(lo, hi, 0x3210u + 0x1111u * o));
    }
}

// All relaxations (s', j), j = 0..jm, of one prefix on the lane's words.
// JB > 0: shifts up to JB bytes, fully unrolled (jm * EB <= JB guaranteed by
// the host); JB == 0: any shift (runtime loop, generic word fetch).
template <int EB, int CH, int JB>
__device__ __forceinline__ void relax_prefix(const Words<CH> &cur, int jm, const LaneMap &lm,
                                             Words<CH> &ae, Words<CH> &ao)
{
#pragma unroll
    for (int t = 0; t < CH; ++t) acc_window<EB>(cur.v[t], cur.v[t], 0, ae.v[t], ao.v[t]);
    if (jm <= 0) return;
    Words<CH> w1, w2;
#pragma unroll
    for (int t = 0; t < CH; ++t) w1.v[t] = word_left(cur, t, 1, lm, 0xffffffffu);
    if (JB == 0 || JB > 4) {
        if (jm * EB > 4) {
#pragma unroll
            for (int t = 0; t < CH; ++t) w2.v[t] = word_left(cur, t, 2, lm, 0xffffffffu);
        }
    }
    if constexpr (JB > 0) {
        // jm is warp-uniform (all groups walk the same prefix): leave the
        // unrolled sequence with a uniform branch instead of predicating the
        // remaining steps
#pragma unroll
        for (int j = 1; j <= JB / EB; ++j) {
            if (j > jm) break;
            {
                const int db = j * EB;
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    if (db <= 4) acc_window<EB>(w1.v[t], cur.v[t], 4 - db, ae.v[t], ao.v[t]);
                    else acc_window<EB>(w2.v[t], w1.v[t], 8 - db, ae.v[t], ao.v[t]);
                }
            }
        }
    } else {
        for (int j = 1; j <= jm; ++j) {
            const int db = j * EB;
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                if (db <= 4) acc_window<EB>(w1.v[t], cur.v[t], 4 - db, ae.v[t], ao.v[t]);
                else if (db <= 8) acc_window<EB>(w2.v[t], w1.v[t], 8 - db, ae.v[t], ao.v[t]);
                else {
                    const int k = (db + 3) >> 2;
                    acc_window<EB>(word_left(cur, t, k, lm, 0xffffffffu), word_left(cur, t, k - 1, lm, 0xffffffffu),
                                   4 * k - db, ae.v[t], ao.v[t]);
                }
            }
        }
    }
}

// u16-lane window of a packed array shifted right by s u16 positions
// (byte shift db = 2s) given the words 1 and 2 to the left.
__device__ __forceinline__ uint32_t lane_shift(const uint32_t w0, const uint32_t w1, const uint32_t w2, int db,
                                               uint32_t prevk_lo, uint32_t prevk_hi, int ok)
{
    if (db == 0) return w0;
    if (db <= 4) return prmt(w1, w0, 0x3210u + 0x1111u * (4 - db));
    if (db <= 8) return prmt(w2, w1, 0x3210u + 0x1111u * (8 - db));
    return prmt(prevk_lo, prevk_hi, 0x3210u + 0x1111u * ok);
}

}  // namespace

// Prefix offsets/Jmax in constant memory: indexed by a warp-uniform loop
// counter they load into uniform registers, so the j-branches are uniform
// (no reconvergence barriers).  One DP is in flight per device (engine lock).
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
    const int np = (int)(meta->nP - 1);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        out->np = np;
        out->pad = 0;
    }
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ((np + 31) & ~31) && i < CP_MAX;
         i += gridDim.x * blockDim.x) {
        if (i < np) {
            const PrefixEntry pe = gpref[1 + i];
            out->oj[i] = make_int2(-(int)((uint64_t)pe.off * eb / 4), pe.jmax);
        } else {
            out->oj[i] = make_int2(0, 0);
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
    const size_t bytes = 8 + 8 * (size_t)((np + 31) & ~31 < CP_MAX ? ((np + 31) & ~31) : CP_MAX);
    return cudaMemcpyToSymbolAsync(c_pref, d_staging, bytes, (size_t)cslot * sizeof(ConstPref),
                                   cudaMemcpyDeviceToDevice, st);
}

template <typename E, int NW, int CH, int JB, bool CPREF, bool SPLIT>
__global__ void __launch_bounds__(256)
row_fill_swar_kernel(E *table, const RowGeom g, const int64_t *__restrict__ rb,
                     const uint64_t *__restrict__ pwa, int64_t pw_stride,
                     const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta, int J0,
                     int rho, int64_t slot_begin, int64_t slot_count, E *compact, int Lg, int nsplit_arg, int cslot)
{
    constexpr int EB = (int)sizeof(E);
    constexpr uint32_t ONES = 0x00010001u;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    // Programmatic dependent launch: let the next row-level's grid start its
    // prologue now; everything before griddepcontrol.wait below reads only data
    // produced before the first fill launch of the DP (prefix table, row index).
    asm volatile("griddepcontrol.launch_dependents;");
    const ConstPref &cp = c_pref[CPREF ? cslot : 0];
    const int np = CPREF ? cp.np : (int)(meta->nP - 1);
    // s_oj[c] = {-off(s') in words, Jmax(s')}: int32 offsets (the host routes
    // tables of 2^31 words or more to the scalar kernel)
    const int npad = (np + 31) & ~31;  // zero-padded: dummy slots never load and have Jmax 0
    int2 *s_oj = reinterpret_cast<int2 *>(smem_raw);
    uint64_t *s_w = reinterpret_cast<uint64_t *>(s_oj + npad);
    for (int i = threadIdx.x; i < npad; i += blockDim.x) {
        if (CPREF) {
            if (i < np) {
#pragma unroll
                for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = gpref[1 + i].w[w];
            }
        } else if (i < np) {
            const PrefixEntry pe = gpref[1 + i];
            // off(s') in words (a multiple of the padded row, hence of 4 bytes)
            const uint64_t offw = (uint64_t)pe.off * EB / 4;
            s_oj[i] = make_int2(-(int)offw, pe.jmax);
#pragma unroll
            for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = pe.w[w];
        } else {
            s_oj[i] = make_int2(0, 0);
        }
    }
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int rpw = 32 / Lg;
    const int grp = lane / Lg;          // grp >= rpw: idle lane
    const int xl = lane - grp * Lg;
    const LaneMap lm{lane, Lg, grp, xl};
    const unsigned gmask = Lg == 32 ? 0xffffffffu : ((1u << Lg) - 1u);
    // nsplit == 1: every warp owns its own rows.  nsplit > 1 (small row-levels):
    // the nsplit warps of a block share one set of rows, each walks every
    // nsplit-th prefix batch, and warp 0 combines the partial minima (shared
    // memory) before the chain -- the per-row latency drops by ~nsplit.
    const int nsplit = SPLIT ? nsplit_arg : 1;
    const int wid = threadIdx.x >> 5;
    const int64_t gw = SPLIT ? (int64_t)blockIdx.x : ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = SPLIT ? (int64_t)gridDim.x : ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int pbase0 = SPLIT ? wid * 32 : 0;  // non-split: a provably uniform prefix index
    const int pstep = SPLIT ? nsplit * 32 : 32;
    uint32_t *s_red = reinterpret_cast<uint32_t *>(s_w + (size_t)NW * np + 1);  // [warp][2][CH][32]
    const int Lw = (int)(g.Wp * EB / 4);  // words per (padded) row
    uint64_t guard[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) guard[w] = g.guard[w];
    // first row set's index entries, loaded before waiting on the previous level
    int64_t nrb = 0;
    uint64_t npw[NW];
    {
        const int64_t slot = gw * rpw + grp;
        const bool ok = grp < rpw && slot < slot_count;
#pragma unroll
        for (int w = 0; w < NW; ++w) npw[w] = ok ? pwa[(int64_t)w * pw_stride + slot_begin + slot] : 0;
        if (ok) nrb = rb[slot_begin + slot];
    }
    asm volatile("griddepcontrol.wait;" ::: "memory");

    // uniform trip count (every warp of the grid runs the same number of row
    // sets; the tail ones are idle) keeps the prefix loop in uniform control
    // flow, so the constant-bank prefix loads and the j-branches are uniform
    const int64_t nsets = (slot_count + rpw - 1) / rpw;
    const int64_t iters = (nsets + nw - 1) / nw;
    for (int64_t it = 0; it < iters; ++it) {
        const int64_t sb = (it * nw + gw) * rpw;
        {
            const int64_t slot = sb + grp;
            const bool rowok = grp < rpw && slot < slot_count;
            int64_t rowbase = nrb;
            uint64_t pw[NW];
#pragma unroll
            for (int w = 0; w < NW; ++w) pw[w] = npw[w];
            {   // prefetch the next row set's index entries
                const int64_t ns = sb + nw * rpw + grp;
                const bool ok = grp < rpw && ns < slot_count;
#pragma unroll
                for (int w = 0; w < NW; ++w) npw[w] = ok ? pwa[(int64_t)w * pw_stride + slot_begin + ns] : 0;
                nrb = ok ? rb[slot_begin + ns] : 0;
            }
            // int32 word index of this lane's first word (the launcher guarantees < 2^31 words)
            const int rw = (int)(rowbase * EB / 4) + xl;
            const uint32_t *tab32 = reinterpret_cast<const uint32_t *>(table);
            bool wok[CH];
#pragma unroll
            for (int t = 0; t < CH; ++t) wok[t] = rowok && (xl + Lg * t) < Lw;

            // ---- cross-row relaxations
            Words<CH> ae, ao;
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                ae.v[t] = 0xffffffffu;
                ao.v[t] = 0xffffffffu;
            }
            for (int base = pbase0; base < np; base += pstep) {
                // dominance mask of prefixes base .. base+31 for this group's row:
                // lane xl tests base + xl + k*Lg, ceil(32/Lg) ballots
                unsigned m = 0;
                for (int k0 = 0; k0 < 32; k0 += Lg) {
                    const int c = base + k0 + xl;
                    bool dom = false;
                    if (rowok && xl + k0 < 32 && c < np) {
                        dom = true;
#pragma unroll
                        for (int w = 0; w < NW; ++w)
                            dom &= (((pw[w] | guard[w]) - s_w[(size_t)w * np + c]) & guard[w]) == guard[w];
                    }
                    const unsigned bal = __ballot_sync(FULL, dom);
                    if (grp < rpw) m |= ((bal >> (grp * Lg)) & gmask) << k0;
                }
                const int cend = ((np - base < 32 ? np - base : 32) + 3) & ~3;
                // 4 prefixes per step: their gathers are issued before any is consumed
                for (int q0 = 0; q0 < cend; q0 += 4) {
                    Words<CH> curq[4];
                    int jmq[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int q = q0 + u;
                        const int2 oj = CPREF ? cp.oj[base + q] : s_oj[base + q];
                        const bool pd = (m >> q) & 1u;
                        jmq[u] = oj.y;
                        const int wi = rw + oj.x;
#pragma unroll
                        for (int t = 0; t < CH; ++t)
                            curq[u].v[t] = (pd && wok[t]) ? __ldg(tab32 + (wi + Lg * t)) : 0xffffffffu;
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) relax_prefix<EB, CH, JB>(curq[u], jmq[u], lm, ae, ao);
                }
            }

            if (SPLIT) {
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    s_red[((wid * 2 + 0) * CH + t) * 32 + lane] = ae.v[t];
                    s_red[((wid * 2 + 1) * CH + t) * 32 + lane] = ao.v[t];
                }
                __syncthreads();
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
            // ---- in-row chain on plain uint16 lanes: opt = 1 + min(acc, opt(x - j))
            // uint8: E holds x = 4w, 4w+2; O holds x = 4w+1, 4w+3.  uint16: E holds 2w, 2w+1.
            Words<CH> oe, oo;
            constexpr uint32_t CFILL = (EB == 1) ? 0x01ff01ffu : 0xfffefffeu;  // "outside the row"
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
            if (rho == 0 && xl == 0) oe.v[0] &= 0xffff0000u;  // OPT(0) = 0
            // one Bellman-Ford step for shift j: ne/no <- min(ne/no, opt(x - j) + 1)
            auto chain_step = [&](int j, const Words<CH> &e1, const Words<CH> &o1, const Words<CH> &e2,
                                  const Words<CH> &o2, Words<CH> &ne, Words<CH> &no) {
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    if constexpr (EB == 1) {
                        // even dest x = 2i: j even -> E shifted j/2; j odd -> O shifted (j+1)/2
                        // odd dest  x = 2i+1: j even -> O shifted j/2; j odd -> E shifted (j-1)/2
                        const bool odd = j & 1;
                        const int sa = odd ? (j + 1) >> 1 : j >> 1;
                        const int sb = odd ? (j - 1) >> 1 : j >> 1;
                        const uint32_t A0 = odd ? oo.v[t] : oe.v[t], A1 = odd ? o1.v[t] : e1.v[t],
                                       A2 = odd ? o2.v[t] : e2.v[t];
                        const uint32_t B0 = odd ? oe.v[t] : oo.v[t], B1 = odd ? e1.v[t] : o1.v[t],
                                       B2 = odd ? e2.v[t] : o2.v[t];
                        uint32_t plo = 0, phi = 0, qlo = 0, qhi = 0;
                        int po = 0, qo = 0;
                        if (JB == 0 && 2 * sa > 8) {
                            const int k = (2 * sa + 3) >> 2;
                            const Words<CH> &AA = odd ? oo : oe;
                            plo = word_left(AA, t, k, lm, CFILL);
                            phi = word_left(AA, t, k - 1, lm, CFILL);
                            po = 4 * k - 2 * sa;
                        }
                        if (JB == 0 && 2 * sb > 8) {
                            const int k = (2 * sb + 3) >> 2;
                            const Words<CH> &BB = odd ? oe : oo;
                            qlo = word_left(BB, t, k, lm, CFILL);
                            qhi = word_left(BB, t, k - 1, lm, CFILL);
                            qo = 4 * k - 2 * sb;
                        }
                        const uint32_t va = lane_shift(A0, A1, A2, 2 * sa, plo, phi, po);
                        const uint32_t vb = lane_shift(B0, B1, B2, 2 * sb, qlo, qhi, qo);
                        ne.v[t] = vmin2(ne.v[t], va + ONES);
                        no.v[t] = vmin2(no.v[t], vb + ONES);
                    } else {
                        uint32_t plo = 0, phi = 0;
                        int po = 0;
                        if (JB == 0 && 2 * j > 8) {
                            const int k = (2 * j + 3) >> 2;
                            plo = word_left(oe, t, k, lm, CFILL);
                            phi = word_left(oe, t, k - 1, lm, CFILL);
                            po = 4 * k - 2 * j;
                        }
                        const uint32_t va = lane_shift(oe.v[t], e1.v[t], e2.v[t], 2 * j, plo, phi, po);
                        ne.v[t] = vmin2(ne.v[t], vmin2(va, 0xfffefffeu) + ONES);
                    }
                }
            };
            // largest u16-lane shift the chain needs: u8 (J0+1)/2, u16 J0 -> bytes
            const int chain_db = EB == 1 ? 2 * ((J0 + 1) >> 1) : 2 * J0;
            bool changed = true;
            while (__any_sync(FULL, changed)) {
                changed = false;
                Words<CH> e1, o1, e2, o2;
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    e1.v[t] = word_left(oe, t, 1, lm, CFILL);
                    o1.v[t] = EB == 1 ? word_left(oo, t, 1, lm, CFILL) : 0u;
                    e2.v[t] = e1.v[t];
                    o2.v[t] = o1.v[t];
                }
                if (chain_db > 4) {
#pragma unroll
                    for (int t = 0; t < CH; ++t) {
                        e2.v[t] = word_left(oe, t, 2, lm, CFILL);
                        o2.v[t] = EB == 1 ? word_left(oo, t, 2, lm, CFILL) : 0u;
                    }
                }
                Words<CH> ne = oe, no = oo;
                if constexpr (JB > 0) {
#pragma unroll
                    for (int j = 1; j <= JB / EB; ++j)
                        if (j <= J0) chain_step(j, e1, o1, e2, o2, ne, no);
                } else {
                    for (int j = 1; j <= J0; ++j) chain_step(j, e1, o1, e2, o2, ne, no);
                }
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    if (wok[t] && (ne.v[t] != oe.v[t] || (EB == 1 && no.v[t] != oo.v[t]))) changed = true;
                    oe.v[t] = ne.v[t];
                    oo.v[t] = no.v[t];
                }
            }
            // ---- store the packed row (padding bytes receive don't-care values)
            uint32_t *out32 = compact ? reinterpret_cast<uint32_t *>(compact + slot * g.Wp)
                                      : reinterpret_cast<uint32_t *>(table + rowbase);
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                if (!wok[t]) continue;
                uint32_t wv;
                if constexpr (EB == 1) wv = prmt(oe.v[t], oo.v[t], 0x6240u);
                else wv = oe.v[t];
                out32[xl + Lg * t] = wv;
            }
            __syncwarp();
            }  // chain + store (warp 0 in split mode)
            if (SPLIT) __syncthreads();  // s_red reused by the next row set
        }
    }
}

// Host launcher body for one (E, NW): returns cudaErrorNotSupported when the
// geometry needs the scalar kernel (row longer than 1 KiB, or shifts beyond one
// chunk).
template <typename E, int NW>
static cudaError_t launch_swar_impl(int e, void *table, const RowGeom &g, const int64_t *rb,
                                 const uint64_t *pw, int64_t pw_stride, const PrefixEntry *d_pref,
                                 const DpMeta *d_meta, int64_t nP_bound, int J0, int rho,
                                 int64_t slot_begin, int64_t slot_count, void *compact_out, int sm_count,
                                 cudaStream_t st, int pdl, int cslot)
{
    if (slot_count <= 0) return cudaSuccess;
    const int Lw = (int)(g.Wp * e / 4);
    if ((g.Wp * e) % 4 != 0 || Lw > 256 || J0 * e > 124) return cudaErrorNotSupported;
    // int32 word offsets: the table (incl. padding) must stay below 2^31 words
    {
        int64_t rows_all = 1;
        for (int i = 0; i < g.K1; ++i) rows_all *= (int64_t)g.N[i] + 1;
        if (rows_all * (int64_t)Lw >= ((int64_t)1 << 31)) return cudaErrorNotSupported;
    }
    // words per lane (chunks, stride Lg) and group width Lg (any 1..32):
    // amortise the per-prefix cost over CH words while leaving few slots idle.
    int CH;
    const char *chs = std::getenv("PTAS_SWAR_CH");
    // small row-levels are latency-bound: fewer words per lane (more lanes per
    // row) shorten each lane's serial work
    const char *cht = std::getenv("PTAS_SMALL_LEVEL_ROWS");
    const int64_t small_rows = cht ? std::atoll(cht) : (int64_t)sm_count * 32;
    if (Lw > 32) CH = Lw <= 64 ? 2 : (Lw <= 128 ? 4 : 8);
    else if (chs && chs[0]) CH = std::atoi(chs);
    else CH = (Lw >= 8 && slot_count > small_rows) ? 2 : 1;
    if (CH != 1 && CH != 2 && CH != 4 && CH != 8) CH = 1;
    int Lg = (Lw + CH - 1) / CH;
    if (Lg < 1) Lg = 1;
    if (Lg > 32) return cudaErrorNotSupported;
    const int rpw = 32 / Lg;
    const int bs = 256;
    int64_t blocks = (slot_count + (int64_t)(bs / 32) * rpw - 1) / ((int64_t)(bs / 32) * rpw);
    const int64_t cap = (int64_t)sm_count * 8;
    if (blocks > cap) blocks = cap;
    // small row-levels: split each row set's prefixes over the 8 warps of a block
    const char *sp = std::getenv("PTAS_SPLIT_ROWS");
    // (prefix batches are 32 wide: splitting pays only with several batches)
    const int64_t np_ = nP_bound > 1 ? nP_bound - 1 : 0;
    const int64_t split_rows = sp ? std::atoll(sp) : (np_ >= 128 ? (int64_t)sm_count * rpw * 2 : 0);
    int nsplit = 1;
    if (slot_count <= split_rows) {
        nsplit = bs / 32;
        blocks = (slot_count + rpw - 1) / rpw;
    }
    const int NWk = NW;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    const size_t smem = (size_t)((np + 31) & ~31) * 8 + (size_t)np * 8 * NWk + 16 + (size_t)(bs / 32) * 2 * 8 * 32 * 4;
    if (smem > 220 * 1024) return cudaErrorNotSupported;
    cudaError_t err;
    // static shift window: chain needs u16-lane shifts up to (J0+1)/2 (u8) or J0 (u16)
    const int need = e == 1 ? ((J0 + 1) / 2 * 2 > J0 ? (J0 + 1) / 2 * 2 : J0) : 2 * J0;
    const int JBsel = need <= 4 ? 4 : (need <= 8 ? 8 : 0);
    const bool cpref = np <= CP_MAX && cslot >= 0 && cslot < CP_SLOTS && np >= 64;
#define PTAS_SWAR_JB(E_, NW_, CH_, JB_)                                                           \
    do {                                                                                          \
        auto kfn = cpref ? (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, JB_, true, true>      \
                                       : row_fill_swar_kernel<E_, NW_, CH_, JB_, true, false>)    \
                         : (nsplit > 1 ? row_fill_swar_kernel<E_, NW_, CH_, JB_, false, true>     \
                                       : row_fill_swar_kernel<E_, NW_, CH_, JB_, false, false>);                                            \
        if (smem > 48 * 1024) {                                                                   \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize,          \
                                       (int)smem);                                                \
            if (err != cudaSuccess) return err;                                                   \
        }                                                                                         \
        cudaLaunchConfig_t cfg = {};                                                              \
        cudaLaunchAttribute attr[1];                                                              \
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;                          \
        attr[0].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;                         \
        cfg.gridDim = dim3((unsigned)blocks);                                                     \
        cfg.blockDim = dim3(bs);                                                                  \
        cfg.dynamicSmemBytes = smem;                                                              \
        cfg.stream = st;                                                                          \
        cfg.attrs = attr;                                                                         \
        cfg.numAttrs = 1;                                                                         \
        err = cudaLaunchKernelEx(&cfg, kfn, (E_ *)table, g, rb, pw, pw_stride, d_pref, d_meta,    \
                                 J0, rho, slot_begin, slot_count, (E_ *)compact_out, Lg,          \
                                 nsplit, cslot);                                                  \
        if (err != cudaSuccess) return err;                                                       \
    } while (0)
#define PTAS_SWAR_CASE(E_, NW_, CH_)                                                              \
    do {                                                                                          \
        if (JBsel == 4) PTAS_SWAR_JB(E_, NW_, CH_, 4);                                            \
        else if (JBsel == 8) PTAS_SWAR_JB(E_, NW_, CH_, 8);                                       \
        else PTAS_SWAR_JB(E_, NW_, CH_, 0);                                                       \
    } while (0)
#define PTAS_SWAR_CH(E_, NW_)                                                                     \
    do {                                                                                          \
        if (CH == 1) PTAS_SWAR_CASE(E_, NW_, 1);                                                  \
        else if (CH == 2) PTAS_SWAR_CASE(E_, NW_, 2);                                             \
        else if (CH == 4) PTAS_SWAR_CASE(E_, NW_, 4);                                             \
        else PTAS_SWAR_CASE(E_, NW_, 8);                                                          \
    } while (0)
    PTAS_SWAR_CH(E, NW);
#undef PTAS_SWAR_CH
#undef PTAS_SWAR_CASE
#undef PTAS_SWAR_JB
    return cudaGetLastError();
}

}  // namespace swar
}  // namespace ptas
