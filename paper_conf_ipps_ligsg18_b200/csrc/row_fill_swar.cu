// row_fill_swar.cu — packed-word level fill, the production kernel of §8(a) a-5.
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
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "internal.h"

namespace ptas {

namespace {

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel)
{
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

__device__ __forceinline__ uint32_t vmin2(uint32_t a, uint32_t b) { return __vminu2(a, b); }

// Word k words to the left of word position (lane xl, chunk t) within a row
// of lane group width Lg (k >= 1).  Source lane (xl - k) mod Lg; lanes that
// wrap supply the previous chunk's word (`prev`, `fill` before chunk 0).
__device__ __forceinline__ uint32_t word_left(uint32_t cur, uint32_t prev, int xl, int k, int Lg)
{
    if (k >= Lg) return prev;  // only reachable for Lg == 32 with k == 32 (caller bounds k)
    const uint32_t send = (xl >= Lg - k) ? prev : cur;
    return __shfl_sync(FULL, send, (xl - k) & (Lg - 1), Lg);
}

template <int CH>
struct Words {
    uint32_t v[CH];
};

}  // namespace

template <typename E, int NW, int CH>
__global__ void __launch_bounds__(256)
row_fill_swar_kernel(E *table, const RowGeom g, const int64_t *__restrict__ gcnt,
                     const PrefixEntry *__restrict__ gpref, const DpMeta *__restrict__ meta, int J0,
                     int rho, int64_t slot_begin, int64_t slot_count, E *compact, int lglog, int crows)
{
    constexpr int EB = (int)sizeof(E);
    constexpr uint32_t ONES = 0x00010001u;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int np = (int)(meta->nP - 1);
    const int ncnt = (g.K1 + 1) * (g.rho_max + 1);
    uint64_t *s_oj = reinterpret_cast<uint64_t *>(smem_raw);
    uint64_t *s_w = s_oj + np;
    int64_t *s_cnt = reinterpret_cast<int64_t *>(s_w + (size_t)NW * np);
    for (int i = threadIdx.x; i < np; i += blockDim.x) {
        const PrefixEntry pe = gpref[1 + i];
        // off(s') in words (a multiple of the padded row, hence of 4 bytes)
        const uint64_t offw = (uint64_t)pe.off * EB / 4;
        s_oj[i] = ((uint64_t)(uint32_t)pe.jmax << 48) | offw;
#pragma unroll
        for (int w = 0; w < NW; ++w) s_w[(size_t)w * np + i] = pe.w[w];
    }
    for (int i = threadIdx.x; i < ncnt; i += blockDim.x) s_cnt[i] = gcnt[i];
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int Lg = 1 << lglog;
    const int grp = lane >> lglog;
    const int xl = lane & (Lg - 1);
    const int rpw = 32 >> lglog;
    const unsigned gmask = Lg == 32 ? 0xffffffffu : ((1u << Lg) - 1u);
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int Lw = (int)(g.Wp * EB / 4);  // words per (padded) row
    const int64_t nchunks = (slot_count + crows - 1) / crows;
    uint64_t guard[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) guard[w] = g.guard[w];
    int32_t d[MAXK];

    for (int64_t cb = gw * rpw; cb < nchunks; cb += nw * rpw) {
        const int64_t ch = cb + grp;
        const int64_t r0 = ch * crows;
        const int64_t r1 = r0 + crows < slot_count ? r0 + crows : slot_count;
        int64_t rowbase = 0;
        uint64_t pw[NW];
#pragma unroll
        for (int w = 0; w < NW; ++w) pw[w] = 0;
        for (int rr = 0; rr < crows; ++rr) {
            const int64_t slot = r0 + rr;
            const bool rowok = slot < r1;
            if (!__any_sync(FULL, rowok)) break;
            if (rowok) {
                if (rr == 0) unrank_digits(g, s_cnt, rho, slot_begin + slot, d);
                else next_in_level(g, d);
                rowbase = 0;
#pragma unroll
                for (int w = 0; w < NW; ++w) pw[w] = 0;
                for (int i = 0; i < g.K1; ++i) {
                    rowbase += (int64_t)d[i] * g.stride[i];
#pragma unroll
                    for (int w = 0; w < NW; ++w)
                        if (g.word[i] == w) pw[w] |= (uint64_t)d[i] << g.shift[i];
                }
            }
            const uint32_t *row32 = reinterpret_cast<const uint32_t *>(table + rowbase) + xl;
            bool wok[CH];
#pragma unroll
            for (int t = 0; t < CH; ++t) wok[t] = rowok && (xl + 32 * t) < Lw;

            // ---- cross-row relaxations
            Words<CH> ae, ao;
#pragma unroll
            for (int t = 0; t < CH; ++t) {
                ae.v[t] = 0xffffffffu;
                ao.v[t] = 0xffffffffu;
            }
            for (int base = 0; base < np; base += Lg) {
                const int c = base + xl;
                bool dom = false;
                if (rowok && c < np) {
                    dom = true;
#pragma unroll
                    for (int w = 0; w < NW; ++w)
                        dom &= (((pw[w] | guard[w]) - s_w[(size_t)w * np + c]) & guard[w]) == guard[w];
                }
                const unsigned m = (__ballot_sync(FULL, dom) >> (grp << lglog)) & gmask;
                const int cend = np - base < Lg ? np - base : Lg;
                // 4 prefixes per step: their gathers are issued before any is consumed
                for (int q0 = 0; q0 < cend; q0 += 4) {
                    Words<CH> curq[4];
                    int jmq[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int q = q0 + u;
                        const bool live = q < cend;
                        const bool pd = live && ((m >> q) & 1u);
                        const uint64_t oj = live ? s_oj[base + q] : 0ull;
                        const uint32_t *src = row32 - (int64_t)(oj & 0xffffffffffffull);
                        jmq[u] = live ? (int)(oj >> 48) : -1;
#pragma unroll
                        for (int t = 0; t < CH; ++t)
                            curq[u].v[t] = (pd && wok[t]) ? src[32 * t] : 0xffffffffu;
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int jm = jmq[u];
                        if (jm < 0) break;
                        const Words<CH> &cur = curq[u];
                        // j = 0: the aligned word itself
#pragma unroll
                        for (int t = 0; t < CH; ++t) {
                            if constexpr (EB == 1) {
                                ae.v[t] = vmin2(ae.v[t], prmt(cur.v[t], cur.v[t], 0xA280u));
                                ao.v[t] = vmin2(ao.v[t], prmt(cur.v[t], cur.v[t], 0xB391u));
                            } else {
                                ae.v[t] = vmin2(ae.v[t], cur.v[t]);
                            }
                        }
                        if (jm == 0) continue;
                        Words<CH> w1, w2;
#pragma unroll
                        for (int t = 0; t < CH; ++t) {
                            const uint32_t prev = t ? cur.v[t - 1] : 0xffffffffu;
                            w1.v[t] = word_left(cur.v[t], prev, xl, 1, Lg);
                        }
                        if (jm * EB > 4) {
#pragma unroll
                            for (int t = 0; t < CH; ++t) {
                                const uint32_t prev = t ? cur.v[t - 1] : 0xffffffffu;
                                w2.v[t] = word_left(cur.v[t], prev, xl, 2, Lg);
                            }
                        }
                        for (int j = 1; j <= jm; ++j) {
                            const int db = j * EB;  // byte shift
#pragma unroll
                            for (int t = 0; t < CH; ++t) {
                                uint32_t lo, hi;
                                int o;
                                if (db <= 4) {
                                    lo = w1.v[t];
                                    hi = cur.v[t];
                                    o = 4 - db;
                                } else if (db <= 8) {
                                    lo = w2.v[t];
                                    hi = w1.v[t];
                                    o = 8 - db;
                                } else {
                                    const int k = (db + 3) >> 2;
                                    const uint32_t prev = t ? cur.v[t - 1] : 0xffffffffu;
                                    lo = word_left(cur.v[t], prev, xl, k, Lg);
                                    hi = word_left(cur.v[t], prev, xl, k - 1, Lg);
                                    o = 4 * k - db;
                                }
                                if constexpr (EB == 1) {
                                    ae.v[t] = vmin2(ae.v[t], prmt(lo, hi, 0xA280u + 0x1111u * o));
                                    ao.v[t] = vmin2(ao.v[t], prmt(lo, hi, 0xB391u + 0x1111u * o));
                                } else {
                                    ae.v[t] = vmin2(ae.v[t], prmt(lo, hi, 0x3210u + 0x1111u * o));
                                }
                            }
                        }
                    }
                }
            }

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
            bool changed = true;
            while (__any_sync(FULL, changed)) {
                changed = false;
                // left neighbour words (1 and 2 back) of both arrays
                Words<CH> e1, o1, e2, o2;
#pragma unroll
                for (int t = 0; t < CH; ++t) {
                    e1.v[t] = word_left(oe.v[t], t ? oe.v[t - 1] : CFILL, xl, 1, Lg);
                    if constexpr (EB == 1) o1.v[t] = word_left(oo.v[t], t ? oo.v[t - 1] : CFILL, xl, 1, Lg);
                }
                const int jl = J0;
                // lanes are shifted by s u16 positions = 2s bytes within (word_left, word)
                if ((EB == 1 && jl > 4) || (EB == 2 && jl > 2)) {
#pragma unroll
                    for (int t = 0; t < CH; ++t) {
                        e2.v[t] = word_left(oe.v[t], t ? oe.v[t - 1] : CFILL, xl, 2, Lg);
                        if constexpr (EB == 1) o2.v[t] = word_left(oo.v[t], t ? oo.v[t - 1] : CFILL, xl, 2, Lg);
                    }
                }
                Words<CH> ne = oe, no = oo;
                for (int j = 1; j <= jl; ++j) {
#pragma unroll
                    for (int t = 0; t < CH; ++t) {
                        if constexpr (EB == 1) {
                            // even dest x = 2i: j even -> E shifted h = j/2; j odd -> O shifted (j+1)/2
                            // odd dest  x = 2i+1: j even -> O shifted j/2;  j odd -> E shifted (j-1)/2
                            const int sa = (j & 1) ? (j + 1) >> 1 : j >> 1;  // shift for even dest
                            const int sb = (j & 1) ? (j - 1) >> 1 : j >> 1;  // shift for odd dest
                            const Words<CH> &A = (j & 1) ? oo : oe;          // source of even dest
                            const Words<CH> &A1 = (j & 1) ? o1 : e1;
                            const Words<CH> &A2 = (j & 1) ? o2 : e2;
                            const Words<CH> &B = (j & 1) ? oe : oo;          // source of odd dest
                            const Words<CH> &B1 = (j & 1) ? e1 : o1;
                            const Words<CH> &B2 = (j & 1) ? e2 : o2;
                            uint32_t va, vb;
                            {
                                const int db = 2 * sa;
                                if (db == 0) va = A.v[t];
                                else if (db <= 4) va = prmt(A1.v[t], A.v[t], 0x3210u + 0x1111u * (4 - db));
                                else if (db <= 8) va = prmt(A2.v[t], A1.v[t], 0x3210u + 0x1111u * (8 - db));
                                else {
                                    const int k = (db + 3) >> 2;
                                    const uint32_t pv = t ? A.v[t - 1] : CFILL;
                                    va = prmt(word_left(A.v[t], pv, xl, k, Lg), word_left(A.v[t], pv, xl, k - 1, Lg),
                                              0x3210u + 0x1111u * (4 * k - db));
                                }
                            }
                            {
                                const int db = 2 * sb;
                                if (db == 0) vb = B.v[t];
                                else if (db <= 4) vb = prmt(B1.v[t], B.v[t], 0x3210u + 0x1111u * (4 - db));
                                else if (db <= 8) vb = prmt(B2.v[t], B1.v[t], 0x3210u + 0x1111u * (8 - db));
                                else {
                                    const int k = (db + 3) >> 2;
                                    const uint32_t pv = t ? B.v[t - 1] : CFILL;
                                    vb = prmt(word_left(B.v[t], pv, xl, k, Lg), word_left(B.v[t], pv, xl, k - 1, Lg),
                                              0x3210u + 0x1111u * (4 * k - db));
                                }
                            }
                            ne.v[t] = vmin2(ne.v[t], va + ONES);
                            no.v[t] = vmin2(no.v[t], vb + ONES);
                        } else {
                            const int db = 2 * j;
                            uint32_t va;
                            if (db <= 4) va = prmt(e1.v[t], oe.v[t], 0x3210u + 0x1111u * (4 - db));
                            else if (db <= 8) va = prmt(e2.v[t], e1.v[t], 0x3210u + 0x1111u * (8 - db));
                            else {
                                const int k = (db + 3) >> 2;
                                const uint32_t pv = t ? oe.v[t - 1] : CFILL;
                                va = prmt(word_left(oe.v[t], pv, xl, k, Lg), word_left(oe.v[t], pv, xl, k - 1, Lg),
                                          0x3210u + 0x1111u * (4 * k - db));
                            }
                            ne.v[t] = vmin2(ne.v[t], vmin2(va, 0xfffefffeu) + ONES);
                        }
                    }
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
                out32[xl + 32 * t] = wv;
            }
            __syncwarp();
        }
    }
}

// Host launcher: returns cudaErrorNotSupported when the geometry needs the
// scalar kernel (row longer than 1 KiB, or shifts beyond one chunk).
cudaError_t launch_row_fill_swar(int e, void *table, const RowGeom &g, const int64_t *d_cnt,
                                 const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound,
                                 int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 void *compact_out, int sm_count, cudaStream_t st)
{
    if (slot_count <= 0) return cudaSuccess;
    const int Lw = (int)(g.Wp * e / 4);
    if ((g.Wp * e) % 4 != 0 || Lw > 256 || J0 * e > 124) return cudaErrorNotSupported;
    int lglog = 0;
    while ((1 << lglog) < Lw && lglog < 5) ++lglog;
    const int Lg = 1 << lglog;
    if (Lw <= 32 && J0 * e > 4 * Lg) {
        // all shifts beyond the row: still correct (INF fill), but keep k < Lg
    }
    const int CH = Lw <= 32 ? 1 : (Lw <= 64 ? 2 : (Lw <= 128 ? 4 : 8));
    const int rpw = 32 >> lglog;
    const int bs = 256;
    const int64_t groups_full = (int64_t)sm_count * 8 * (bs / 32) * rpw;
    int64_t crows = (slot_count + groups_full - 1) / groups_full;  // one unrank per group, then successors
    if (crows < 1) crows = 1;
    if (crows > 32) crows = 32;
    const int64_t nchunks = (slot_count + crows - 1) / crows;
    int64_t blocks = (nchunks + (int64_t)(bs / 32) * rpw - 1) / ((int64_t)(bs / 32) * rpw);
    const int64_t cap = (int64_t)sm_count * 8;
    if (blocks > cap) blocks = cap;
    const int NWk = g.nwords <= 1 ? 1 : 2;
    const int64_t np = nP_bound > 1 ? nP_bound - 1 : 0;
    const size_t smem = (size_t)np * (8 + 8 * NWk) + (size_t)(g.K1 + 1) * (g.rho_max + 1) * 8 + 16;
    if (smem > 220 * 1024) return cudaErrorNotSupported;
    cudaError_t err;
#define PTAS_SWAR_CASE(E_, NW_, CH_)                                                              \
    do {                                                                                          \
        auto kfn = row_fill_swar_kernel<E_, NW_, CH_>;                                            \
        if (smem > 48 * 1024) {                                                                   \
            err = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize,          \
                                       (int)smem);                                                \
            if (err != cudaSuccess) return err;                                                   \
        }                                                                                         \
        kfn<<<(unsigned)blocks, bs, smem, st>>>((E_ *)table, g, d_cnt, d_pref, d_meta, J0, rho,   \
                                                slot_begin, slot_count, (E_ *)compact_out, lglog, \
                                                (int)crows);                                      \
    } while (0)
#define PTAS_SWAR_CH(E_, NW_)                                                                     \
    do {                                                                                          \
        if (CH == 1) PTAS_SWAR_CASE(E_, NW_, 1);                                                  \
        else if (CH == 2) PTAS_SWAR_CASE(E_, NW_, 2);                                             \
        else if (CH == 4) PTAS_SWAR_CASE(E_, NW_, 4);                                             \
        else PTAS_SWAR_CASE(E_, NW_, 8);                                                          \
    } while (0)
    if (e == 1) {
        if (NWk == 1) PTAS_SWAR_CH(uint8_t, 1); else PTAS_SWAR_CH(uint8_t, 2);
    } else {
        if (NWk == 1) PTAS_SWAR_CH(uint16_t, 1); else PTAS_SWAR_CH(uint16_t, 2);
    }
#undef PTAS_SWAR_CH
#undef PTAS_SWAR_CASE
    return cudaGetLastError();
}

}  // namespace ptas
