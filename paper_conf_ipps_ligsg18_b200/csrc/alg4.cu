// alg4.cu — the paper's own data-partitioning scheme (Alg 4 / Alg 5,
// PAPER.md:209-283, 288-338, §III-C/D) rebuilt on B200 as an A/B baseline of
// SURVEY.md §8(f)-3 ("does the paper's data-partitioning help on Blackwell?").
//
//   Alg 4 l.4-10   divisor: per dimension div_i = floor(sqrt(n_i + 1)), lowered
//                  until it divides n_i + 1; only the `dim` largest divisors are
//                  kept (the others set to 1)
//   Alg 4 l.12-19  blocks of bs_i = (n_i + 1) / div_i entries per dimension,
//                  grouped into block-levels (sum of the block coordinates)
//   Alg 4 l.20-28  memory layout: the entries of a block consecutive (row-major
//                  inside the block), blocks in row-major block order:
//                  M(c) = block(c) * jobsPerBlock + inblock(c)
//   Alg 4 l.29-31  block-levels in order, the blocks of one level concurrently
//   Alg 5          inside a block, its anti-diagonal levels in order, the entries
//                  of one level in parallel, each entry relaxed over every
//                  configuration s <= v (Eq. 1)
//
// What is B200-native here (the A/B keeps the paper's layout and schedule, not
// its Kepler mechanics): the blocks of a block-level are ONE grid (one CTA per
// block) instead of one kernel per block cycled over 4 streams; the in-block
// levels are separated by __syncthreads instead of CDP child launches with a
// device-side cudaDeviceSynchronize (removed in CUDA 12); the sub-configuration
// is located by the blocked address M(c - s) = sum_i contrib_i[c_i - s_i]
// (per-digit tables in shared memory) instead of the search of Alg 5 l.26-28.
// Values are bit-identical to the plain recurrence (tests/test_gpu_alg4.py).
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/ptas.h"
#include "internal.h"

namespace ptas {
namespace {

constexpr int A4_MAXK = 16;

struct Alg4Geom {
    int32_t K;
    int32_t nC;
    int32_t div[A4_MAXK];      // blocks per dimension
    int32_t bs[A4_MAXK];       // entries per block per dimension
    int32_t coff[A4_MAXK];     // offset of dimension i's contribution table (entries)
    int64_t jobs_per_block;
    int32_t inb_levels;        // in-block anti-diagonal levels = sum (bs_i - 1) + 1
    int32_t ctab_len;          // sum (n_i + 1)
};

// One block-level: CTA = one block; in-block levels in order.
template <typename E>
__global__ void __launch_bounds__(1024)
alg4_block_kernel(E *__restrict__ table, const Alg4Geom g, const int64_t *__restrict__ ctab_g,
                  const uint16_t *__restrict__ cfg, const int32_t *__restrict__ blocks,
                  const int32_t *__restrict__ inb_order, const int32_t *__restrict__ inb_lstart)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int64_t *ctab = reinterpret_cast<int64_t *>(smem_raw);                       // [ctab_len]
    uint16_t *scfg = reinterpret_cast<uint16_t *>(ctab + g.ctab_len);            // [nC * K]
    for (int i = threadIdx.x; i < g.ctab_len; i += blockDim.x) ctab[i] = ctab_g[i];
    for (int i = threadIdx.x; i < g.nC * g.K; i += blockDim.x) scfg[i] = cfg[i];
    // this CTA's block: coordinates from its row-major block index
    const int32_t bid = blocks[blockIdx.x];
    int32_t bc[A4_MAXK];
    {
        int32_t rem = bid;
        for (int i = g.K - 1; i >= 0; --i) {
            bc[i] = rem % g.div[i];
            rem /= g.div[i];
        }
    }
    __syncthreads();
    for (int l = 0; l < g.inb_levels; ++l) {
        for (int32_t t = inb_lstart[l] + threadIdx.x; t < inb_lstart[l + 1]; t += blockDim.x) {
            // entry of the block: in-block row-major offset -> digits c
            int32_t c[A4_MAXK];
            int32_t rem = inb_order[t];
            bool zero = true;
            for (int i = g.K - 1; i >= 0; --i) {
                c[i] = bc[i] * g.bs[i] + rem % g.bs[i];
                rem /= g.bs[i];
                zero &= c[i] == 0;
            }
            int64_t me = 0;
            for (int i = 0; i < g.K; ++i) me += ctab[g.coff[i] + c[i]];
            int best = 1 << 28;
            if (!zero) {
                for (int q = 0; q < g.nC; ++q) {   // every configuration s <= c (Eq. 1)
                    const uint16_t *s = scfg + q * g.K;
                    bool dom = true;
                    int64_t src = 0;
                    for (int i = 0; i < g.K; ++i) {
                        dom &= s[i] <= c[i];
                        src += dom ? ctab[g.coff[i] + c[i] - s[i]] : 0;
                    }
                    if (dom) {
                        const int v = table[src];
                        best = v < best ? v : best;
                    }
                }
            }
            table[me] = (E)(zero ? 0 : best + 1);
        }
        __syncthreads();   // in-block level l complete (Alg 5 l.9)
    }
}

// blocked -> row-major copy (the caller's layout)
template <typename E>
__global__ void alg4_to_rowmajor_kernel(const E *__restrict__ blocked, E *__restrict__ out, int64_t sigma,
                                        const Alg4Geom g, const int64_t *__restrict__ ctab, const int32_t *__restrict__ N)
{
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < sigma;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int64_t rem = idx, m = 0;
        for (int i = g.K - 1; i >= 0; --i) {
            const int64_t d = rem % (N[i] + 1);
            rem /= N[i] + 1;
            m += ctab[g.coff[i] + d];
        }
        out[idx] = blocked[m];
    }
}

}  // namespace

// Host driver of the A/B (called by dp_fill_alg4, ptas_api.cpp).  cfg_digits:
// C(T) in the caller's class order (host, [nC][K]).  Allocates per call.
int alg4_fill(int e, const int32_t *N, int K, const int32_t *cfg_digits, int64_t nC, int dim, void *host_out,
              int32_t *opt_out, double *fill_s, int64_t *nblocks_out, int32_t *block_levels_out, int32_t *div_out)
{
    if (K < 1 || K > A4_MAXK || nC < 1 || nC > 65535 || dim < 1) return PTAS_EINVAL;
    Alg4Geom g;
    std::memset(&g, 0, sizeof(g));
    g.K = K;
    g.nC = (int32_t)nC;
    // Alg 4 l.4-10: divisor
    std::vector<int32_t> div(K);
    for (int i = 0; i < K; ++i) {
        int32_t d = (int32_t)std::floor(std::sqrt((double)N[i] + 1.0));
        while (d > 1 && (N[i] + 1) % d != 0) --d;
        div[i] = std::max(d, 1);
    }
    std::vector<int> idx(K);
    for (int i = 0; i < K; ++i) idx[i] = i;
    std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return div[a] > div[b]; });
    for (int j = dim; j < K; ++j) div[idx[j]] = 1;
    int64_t nblocks = 1, jpb = 1, sigma = 1;
    int inb_levels = 1, blk_levels = 1;
    for (int i = 0; i < K; ++i) {
        g.div[i] = div[i];
        g.bs[i] = (N[i] + 1) / div[i];
        nblocks *= div[i];
        jpb *= g.bs[i];
        sigma *= N[i] + 1;
        inb_levels += g.bs[i] - 1;
        blk_levels += div[i] - 1;
        if (div_out) div_out[i] = div[i];
    }
    g.jobs_per_block = jpb;
    g.inb_levels = inb_levels;
    // per-digit contribution tables: M(c) = sum_i ctab_i[c_i]
    std::vector<int64_t> ctab;
    {
        std::vector<int64_t> bstride(K, 1), istride(K, 1);
        for (int i = K - 2; i >= 0; --i) {
            bstride[i] = bstride[i + 1] * div[i + 1];
            istride[i] = istride[i + 1] * g.bs[i + 1];
        }
        for (int i = 0; i < K; ++i) {
            g.coff[i] = (int32_t)ctab.size();
            for (int d = 0; d <= N[i]; ++d)
                ctab.push_back((int64_t)(d / g.bs[i]) * bstride[i] * jpb + (int64_t)(d % g.bs[i]) * istride[i]);
        }
        g.ctab_len = (int32_t)ctab.size();
    }
    // Alg 4 l.13-15: blocks by block-level; in-block entries by in-block level
    std::vector<std::vector<int32_t>> by_lvl(blk_levels);
    for (int64_t b = 0; b < nblocks; ++b) {
        int64_t rem = b;
        int lv = 0;
        for (int i = K - 1; i >= 0; --i) {
            lv += (int)(rem % div[i]);
            rem /= div[i];
        }
        by_lvl[lv].push_back((int32_t)b);
    }
    std::vector<int32_t> blocks, blk_lstart(1, 0);
    for (auto &v : by_lvl) {
        blocks.insert(blocks.end(), v.begin(), v.end());
        blk_lstart.push_back((int32_t)blocks.size());
    }
    std::vector<std::vector<int32_t>> inb(inb_levels);
    for (int64_t t = 0; t < jpb; ++t) {
        int64_t rem = t;
        int lv = 0;
        for (int i = K - 1; i >= 0; --i) {
            lv += (int)(rem % g.bs[i]);
            rem /= g.bs[i];
        }
        inb[lv].push_back((int32_t)t);
    }
    std::vector<int32_t> inb_order, inb_lstart(1, 0);
    for (auto &v : inb) {
        inb_order.insert(inb_order.end(), v.begin(), v.end());
        inb_lstart.push_back((int32_t)inb_order.size());
    }
    std::vector<uint16_t> cfg((size_t)nC * K);
    for (size_t i = 0; i < cfg.size(); ++i) cfg[i] = (uint16_t)cfg_digits[i];
    const size_t smem = (size_t)g.ctab_len * 8 + cfg.size() * 2 + 16;
    if (smem > 200 * 1024 || jpb > ((int64_t)1 << 31)) return PTAS_ETOOBIG;

    void *d_table = nullptr, *d_out = nullptr;
    int64_t *d_ctab = nullptr;
    uint16_t *d_cfg = nullptr;
    int32_t *d_blocks = nullptr, *d_inb = nullptr, *d_inbl = nullptr, *d_N = nullptr;
    int rc = PTAS_OK;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    auto ck = [&](cudaError_t x) {
        if (x != cudaSuccess && rc == PTAS_OK) rc = x == cudaErrorMemoryAllocation ? PTAS_ENOMEM : PTAS_ECUDA;
        return rc == PTAS_OK;
    };
    if (ck(cudaMalloc(&d_table, (size_t)sigma * e)) && ck(cudaMalloc(&d_ctab, ctab.size() * 8)) &&
        ck(cudaMalloc(&d_cfg, cfg.size() * 2)) && ck(cudaMalloc(&d_blocks, blocks.size() * 4)) &&
        ck(cudaMalloc(&d_inb, inb_order.size() * 4)) && ck(cudaMalloc(&d_inbl, inb_lstart.size() * 4)) &&
        ck(cudaMalloc(&d_N, (size_t)K * 4)) && ck(cudaMemcpy(d_ctab, ctab.data(), ctab.size() * 8, cudaMemcpyHostToDevice)) &&
        ck(cudaMemcpy(d_cfg, cfg.data(), cfg.size() * 2, cudaMemcpyHostToDevice)) &&
        ck(cudaMemcpy(d_blocks, blocks.data(), blocks.size() * 4, cudaMemcpyHostToDevice)) &&
        ck(cudaMemcpy(d_inb, inb_order.data(), inb_order.size() * 4, cudaMemcpyHostToDevice)) &&
        ck(cudaMemcpy(d_inbl, inb_lstart.data(), inb_lstart.size() * 4, cudaMemcpyHostToDevice)) &&
        ck(cudaMemcpy(d_N, N, (size_t)K * 4, cudaMemcpyHostToDevice)) && ck(cudaEventCreate(&ev0)) &&
        ck(cudaEventCreate(&ev1))) {
        auto kfn = e == 1 ? (void *)alg4_block_kernel<uint8_t> : (void *)alg4_block_kernel<uint16_t>;
        ck(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        ck(cudaEventRecord(ev0));
        for (int lv = 0; lv < blk_levels && rc == PTAS_OK; ++lv) {   // Alg 4 l.29-31
            const int nb = blk_lstart[lv + 1] - blk_lstart[lv];
            if (nb <= 0) continue;
            if (e == 1)
                alg4_block_kernel<uint8_t><<<nb, 1024, smem>>>((uint8_t *)d_table, g, d_ctab, d_cfg,
                                                                d_blocks + blk_lstart[lv], d_inb, d_inbl);
            else
                alg4_block_kernel<uint16_t><<<nb, 1024, smem>>>((uint16_t *)d_table, g, d_ctab, d_cfg,
                                                                 d_blocks + blk_lstart[lv], d_inb, d_inbl);
            ck(cudaGetLastError());
        }
        ck(cudaEventRecord(ev1));
        ck(cudaEventSynchronize(ev1));
        float ms = 0;
        ck(cudaEventElapsedTime(&ms, ev0, ev1));
        if (fill_s) *fill_s = ms * 1e-3;
        // OPT(N) at M(N)
        int64_t mN = 0;
        for (int i = 0; i < K; ++i) mN += ctab[g.coff[i] + N[i]];
        uint16_t v = 0;
        ck(cudaMemcpy(&v, (unsigned char *)d_table + mN * e, e, cudaMemcpyDeviceToHost));
        if (rc == PTAS_OK) *opt_out = e == 1 ? (int32_t)(v & 0xff) : (int32_t)v;
        if (host_out && rc == PTAS_OK && ck(cudaMalloc(&d_out, (size_t)sigma * e))) {
            if (e == 1)
                alg4_to_rowmajor_kernel<uint8_t><<<1184, 256>>>((const uint8_t *)d_table, (uint8_t *)d_out, sigma, g,
                                                                d_ctab, d_N);
            else
                alg4_to_rowmajor_kernel<uint16_t><<<1184, 256>>>((const uint16_t *)d_table, (uint16_t *)d_out, sigma, g,
                                                                 d_ctab, d_N);
            ck(cudaGetLastError());
            ck(cudaMemcpy(host_out, d_out, (size_t)sigma * e, cudaMemcpyDeviceToHost));
        }
    }
    cudaFree(d_table);
    cudaFree(d_out);
    cudaFree(d_ctab);
    cudaFree(d_cfg);
    cudaFree(d_blocks);
    cudaFree(d_inb);
    cudaFree(d_inbl);
    cudaFree(d_N);
    if (ev0) cudaEventDestroy(ev0);
    if (ev1) cudaEventDestroy(ev1);
    if (nblocks_out) *nblocks_out = nblocks;
    if (block_levels_out) *block_levels_out = blk_levels;
    cudaGetLastError();
    return rc;
}

}  // namespace ptas
