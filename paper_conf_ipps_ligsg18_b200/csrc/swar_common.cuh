// swar_common.cuh — packed-word (SWAR) helpers shared by the level-fill
// kernels (row_fill_swar.cuh, row_ring.cu): lane-chunk loads/stores, the
// shifted prefix windows of reading D5 built with shuffles + PRMT, and the
// kernel-side prefix entry.  Product only (never used by oracle/).
#pragma once
#include <cstdint>
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

template <int CH>
__device__ __forceinline__ void fill_words(Words<CH> &w, uint32_t x)
{
#pragma unroll
    for (int t = 0; t < CH; ++t) w.v[t] = x;
}

#ifndef PTAS_DF_NOACQ
#define PTAS_DF_NOACQ 0
#endif
#ifndef PTAS_DF_PROFILE
#define PTAS_DF_PROFILE 0
#endif
#ifndef PTAS_DF_LD_CG
#define PTAS_DF_LD_CG 0
#endif
// Coherent 32-bit loads of table words for the dataflow kernel (the table is
// written during the launch, so the read-only path is not allowed): ordinary
// weak loads, kept after the flag acquire by `volatile` (the acquire
// invalidates L1); PTAS_DF_LD_CG=1 reads through L2 only.
__device__ __forceinline__ uint32_t ld_co(const uint32_t *p)
{
    uint32_t v;
    if (PTAS_DF_LD_CG) asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else asm volatile("ld.global.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint2 ld_co2(const uint32_t *p)
{
    uint2 v;
    if (PTAS_DF_LD_CG) asm volatile("ld.global.cg.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p));
    else asm volatile("ld.global.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p));
    return v;
}
__device__ __forceinline__ uint4 ld_co4(const uint32_t *p)
{
    uint4 v;
    if (PTAS_DF_LD_CG)
        asm volatile("ld.global.cg.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else
        asm volatile("ld.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint32_t *p, uint32_t v)
{
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// CH consecutive words at p (4*CH-byte aligned: the pitch is a multiple of CH words)
template <int CH, bool CO = false>
__device__ __forceinline__ Words<CH> load_words(const uint32_t *p)
{
    Words<CH> w;
    if constexpr (CO) {
        if constexpr (CH == 1) {
            w.v[0] = ld_co(p);
        } else if constexpr (CH == 2) {
            const uint2 a = ld_co2(p);
            w.v[0] = a.x;
            w.v[1] = a.y;
        } else {
#pragma unroll
            for (int c = 0; c < CH; c += 4) {
                const uint4 a = ld_co4(p + c);
                w.v[c] = a.x;
                w.v[c + 1] = a.y;
                w.v[c + 2] = a.z;
                w.v[c + 3] = a.w;
            }
        }
    } else if constexpr (CH == 1) {
        w.v[0] = __ldg(p);
    } else if constexpr (CH == 2) {
        const uint2 a = __ldg(reinterpret_cast<const uint2 *>(p));
        w.v[0] = a.x;
        w.v[1] = a.y;
    } else {
#pragma unroll
        for (int c = 0; c < CH; c += 4) {
            const uint4 a = __ldg(reinterpret_cast<const uint4 *>(p + c));
            w.v[c] = a.x;
            w.v[c + 1] = a.y;
            w.v[c + 2] = a.z;
            w.v[c + 3] = a.w;
        }
    }
    return w;
}

template <int CH>
__device__ __forceinline__ void store_words(uint32_t *p, const Words<CH> &w)
{
    if constexpr (CH == 1) {
        p[0] = w.v[0];
    } else if constexpr (CH == 2) {
        *reinterpret_cast<uint2 *>(p) = make_uint2(w.v[0], w.v[1]);
    } else {
#pragma unroll
        for (int c = 0; c < CH; c += 4)
            *reinterpret_cast<uint4 *>(p + c) = make_uint4(w.v[c], w.v[c + 1], w.v[c + 2], w.v[c + 3]);
    }
}

// Word w - k of the row for the lane's slot t (w = xl*CH + t), k >= 0 warp-uniform;
// `fill` for w - k < 0.  Every lane of the warp must call it (shuffle).
template <int CH>
__device__ __forceinline__ uint32_t word_back(const Words<CH> &a, int t, int k, int xl, uint32_t fill)
{
    const int d = k - t;  // > 0: the word lives in a lane to the left
    if (d <= 0) {
        uint32_t r = a.v[0];
#pragma unroll
        for (int c = 1; c < CH; ++c)
            if (c == t - k) r = a.v[c];
        return r;
    }
    const int dl = (d + CH - 1) / CH;
    const int slot = dl * CH - d;
    uint32_t send = a.v[0];
#pragma unroll
    for (int c = 1; c < CH; ++c)
        if (c == slot) send = a.v[c];
    const uint32_t got = __shfl_up_sync(FULL, send, dl > 31 ? 31 : dl);
    return xl >= dl ? got : fill;
}

// Operands of the 4-byte window that starts db bytes left of each of the
// lane's words: PRMT(lo, hi) at byte offset o = (4 - db % 4) % 4, with
// lo = word w - k1, hi = word w - k1 + 1, k1 = ceil(db / 4) (db > 0; the
// caller uses the word itself for db = 0).  db <= 4: the only word needed
// from another lane is the left neighbour's last one (one shuffle); db <= 8:
// two shuffles; longer shifts: word_back.  WIN = the largest db the caller
// can pass (4, 8, or 0 = any), so the unneeded forms are not compiled.  Words before
// the row read `fill`.
template <int CH, int WIN>
__device__ __forceinline__ void windows(const Words<CH> &a, int db, int xl, uint32_t fill, Words<CH> &lo,
                                        Words<CH> &hi)
{
    const uint32_t left = __shfl_up_sync(FULL, a.v[CH - 1], 1);
    const uint32_t l1 = xl >= 1 ? left : fill;   // word w - 1 of slot 0
    if (WIN == 4 || db <= 4) {
#pragma unroll
        for (int t = 0; t < CH; ++t) {
            lo.v[t] = t == 0 ? l1 : a.v[t - 1];
            hi.v[t] = a.v[t];
        }
    } else if (WIN == 8 || db <= 8) {
        // word w - 2 of slot 0: lane xl-1's slot CH-2 (CH >= 2) or lane xl-2 (CH = 1)
        const uint32_t left2 = __shfl_up_sync(FULL, a.v[CH >= 2 ? CH - 2 : 0], CH >= 2 ? 1 : 2);
        const uint32_t l2 = xl >= (CH >= 2 ? 1 : 2) ? left2 : fill;
        const bool two = db > 4;   // k1 = 2
#pragma unroll
        for (int t = 0; t < CH; ++t) {
            const uint32_t w1 = t == 0 ? l1 : a.v[t - 1];
            const uint32_t w2 = t >= 2 ? a.v[t - 2] : (t == 1 ? l1 : l2);
            lo.v[t] = two ? w2 : w1;
            hi.v[t] = two ? w1 : a.v[t];
        }
    } else {
        const int k1 = (db + 3) >> 2;
#pragma unroll
        for (int t = 0; t < CH; ++t) {
            lo.v[t] = word_back(a, t, k1, xl, fill);
            hi.v[t] = word_back(a, t, k1 - 1, xl, fill);
        }
    }
}

// Same operands from a copy of the group's row in shared memory (row word r
// at srow[r]), any db > 0: used by the in-row closure's long shifts.
template <int CH>
__device__ __forceinline__ void windows_smem(const uint32_t *srow, int db, int xl, uint32_t fill, Words<CH> &lo,
                                             Words<CH> &hi)
{
    const int k1 = (db + 3) >> 2;
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int w = xl * CH + t - k1;
        lo.v[t] = w >= 0 ? srow[w] : fill;
        hi.v[t] = w + 1 >= 0 ? srow[w + 1] : fill;
    }
}

// Kernel-side prefix entry: x = -off(s') in words, y = PRMT selector of the
// window (low 16 bits; the odd-byte selector is y + 0x1111) | db << 16, where
// db = Jmax(s') * e is the window's byte shift.  db = 0 (the word itself)
// takes byte offset 4, i.e. the selector reads the high operand (the word)
// only, so every prefix runs the same branch-free window code.
constexpr int SEL_U8 = 0xA280, SEL_U16 = 0x3210, SEL_SELF = 0x4444;
__device__ __forceinline__ int2 oj_entry(const PrefixEntry &pe, int eb)
{
    const int db = pe.jmax * eb;
    const int o = db == 0 ? 4 : (4 - (db & 3)) & 3;
    const int sel = (eb == 1 ? SEL_U8 : SEL_U16) + 0x1111 * o;
    return make_int2(-(int)((uint64_t)pe.off * eb / 4), sel | (db << 16));
}

}  // namespace

}  // namespace swar
}  // namespace ptas
