// dp_engine.cpp — per-device orchestration of one DP(N, T) on the GPU.
//
// One DP = §8(a) rows a-2 .. a-6:
//   a-2 table geometry, budget guard (host, O(K))
//   a-3 enum_configs (2 passes + scan) and build_prefix kernels
//   a-4 row-level sizes = coefficients of prod_{i<K-1} (1 + z + ... + z^{N_i})
//       (host, the cnt[] suffix-count table, uploaded once) + on-device
//       unranking inside the fill kernels
//   a-5 one row_fill launch per row-level rho = 0 .. sum_{i<K-1} N_i
//       (optionally sharded: compact slice -> NCCL all-gather -> scatter)
//   a-6 OPT(N) read back with the planning summary in one 40-byte D2H.
// Host syncs per DP: one after the config count (to size C), one at the end.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <numeric>

#include <cuda.h>

#include "engine.h"

namespace ptas {

// PTAS_SLOW_CALLS=<ms> (diagnostics): report every checked call slower than
// <ms> milliseconds of host time, with its source line.
static double slow_call_ms()
{
    static const double v = [] {
        const char *t = std::getenv("PTAS_SLOW_CALLS");
        return t ? std::atof(t) : 0.0;
    }();
    return v;
}
static double host_ms()
{
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
#define PT_CK(x)                                                                   \
    do {                                                                           \
        const double t0__ = slow_call_ms() > 0 ? host_ms() : 0.0;                  \
        cudaError_t e__ = (x);                                                     \
        if (t0__ > 0 && host_ms() - t0__ > slow_call_ms())                         \
            std::fprintf(stderr, "[ptas] slow call %.2f ms at dp_engine.cpp:%d: %s\n", \
                         host_ms() - t0__, __LINE__, #x);                            \
        if (e__ != cudaSuccess) {                                                  \
            std::fprintf(stderr, "[ptas] CUDA error at dp_engine.cpp:%d: %s: %s\n", __LINE__, #x, \
                         cudaGetErrorString(e__));                                 \
            cudaGetLastError();                                                    \
            return e__ == cudaErrorMemoryAllocation ? PTAS_ENOMEM : PTAS_ECUDA;    \
        }                                                                          \
    } while (0)

cudaError_t DpSlot::Buf::ensure(size_t bytes)
{
    if (p && bytes <= cap) return cudaSuccess;
    if (p) {
        cudaFree(p);
        p = nullptr;
        cap = 0;
    }
    size_t want = bytes < 256 ? 256 : bytes;
    cudaError_t e = cudaMalloc(&p, want);
    if (e != cudaSuccess) {
        p = nullptr;
        cap = 0;
        cudaGetLastError();
        return e;
    }
    cap = want;
    return cudaSuccess;
}

static std::mutex g_reg_mu;
static std::map<int, Engine *> g_engines;

int Engine::get(int device, Engine **out)
{
    std::lock_guard<std::mutex> lk(g_reg_mu);
    auto it = g_engines.find(device);
    if (it != g_engines.end()) {
        *out = it->second;
        return PTAS_OK;
    }
    Engine *e = new Engine();
    int rc = e->init(device);
    if (rc) {
        delete e;
        return rc;
    }
    g_engines[device] = e;
    *out = e;
    return PTAS_OK;
}

// The host driver waits for small readbacks many times per solve; a spin on
// an event query avoids the scheduler wake-up latency of a blocking sync.
cudaError_t DpSlot::sync_spin(cudaStream_t st)
{
    cudaError_t e = cudaEventRecord(ev_sync_, st);
    if (e != cudaSuccess) return e;
    for (;;) {
        e = cudaEventQuery(ev_sync_);
        if (e != cudaErrorNotReady) return e;
    }
}

cudaError_t DpSlot::h2d(void *dst, const void *src, size_t bytes, cudaStream_t st)
{
    const size_t need = (pin_used_ + bytes + 255) & ~(size_t)255;
    if (need > pin_cap_) return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, st);
    unsigned char *h = pin_ + pin_used_;
    std::memcpy(h, src, bytes);
    pin_used_ = need;
    return cudaMemcpyAsync(dst, h, bytes, cudaMemcpyHostToDevice, st);
}

int Engine::init(int device)
{
    device_ = device;
    PT_CK(cudaSetDevice(device));
    PT_CK(cudaDeviceGetAttribute(&sm_count_, cudaDevAttrMultiProcessorCount, device));
    DpSlot *s = nullptr;
    return slot(0, &s);
}

int Engine::mark_reference(cudaStream_t st, cudaEvent_t *out)
{
    if (!ref_ev_) PT_CK(cudaEventCreate(&ref_ev_));
    PT_CK(cudaEventRecord(ref_ev_, st ? st : stream()));
    PT_CK(cudaEventSynchronize(ref_ev_));
    *out = ref_ev_;
    return PTAS_OK;
}

int Engine::slot(int i, DpSlot **out)
{
    if (i < 0 || i >= MAX_SLOTS) return PTAS_EINVAL;
    if (!slots_[i]) {
        DpSlot *s = new DpSlot();
        int rc = s->init(device_, sm_count_, i);
        if (rc) {
            delete s;
            return rc;
        }
        slots_[i] = s;
    }
    *out = slots_[i];
    return PTAS_OK;
}

int DpSlot::init(int device, int sm_count, int index)
{
    device_ = device;
    sm_count_ = sm_count;
    index_ = index;
    PT_CK(cudaSetDevice(device));
    PT_CK(cudaStreamCreateWithFlags(&stream_, cudaStreamNonBlocking));
    for (auto &ev : ev_) PT_CK(cudaEventCreate(&ev));
    PT_CK(cudaEventCreateWithFlags(&ev_sync_, cudaEventDisableTiming));
    PT_CK(cudaStreamCreateWithFlags(&side_, cudaStreamNonBlocking));
    PT_CK(cudaEventCreateWithFlags(&ev_fork_, cudaEventDisableTiming));
    PT_CK(cudaEventCreateWithFlags(&ev_join_, cudaEventDisableTiming));
    PT_CK(cudaMalloc(&d_meta_, sizeof(DpMeta)));
    PT_CK(cudaMallocHost(&h_meta_, sizeof(DpMeta)));
    PT_CK(cudaMallocHost(&h_scalar_, 64));
    pin_cap_ = (size_t)8 << 20;
    PT_CK(cudaMallocHost((void **)&pin_, pin_cap_));
    return PTAS_OK;
}

int64_t DpSlot::free_budget()
{
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    int64_t b = (int64_t)fr + (int64_t)table_.cap - ((int64_t)2 << 30);
    return b > 0 ? b : 0;
}

// ---- level-window ring (D15): `phys` bytes of device memory mapped
// twice, back to back, into one 2 * phys virtual range (CUDA virtual memory
// management, driver entry points fetched through the runtime), so a slab at
// ring position Rw + (p0 mod Rw) sees the slabs p0 - s0 (s0 <= hi0 < Rw) at plain
// negative offsets -- the fill kernels address the window as an ordinary table.
namespace {
struct VmmApi {
    bool ok = false;
    decltype(&cuMemGetAllocationGranularity) gran = nullptr;
    decltype(&cuMemCreate) create = nullptr;
    decltype(&cuMemRelease) release = nullptr;
    decltype(&cuMemAddressReserve) reserve = nullptr;
    decltype(&cuMemAddressFree) addr_free = nullptr;
    decltype(&cuMemMap) map = nullptr;
    decltype(&cuMemUnmap) unmap = nullptr;
    decltype(&cuMemSetAccess) access = nullptr;
};
VmmApi *vmm()
{
    static VmmApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        auto get = [](const char *n, void **f) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(n, f, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *f;
        };
        api.ok = get("cuMemGetAllocationGranularity", (void **)&api.gran) && get("cuMemCreate", (void **)&api.create) &&
                 get("cuMemRelease", (void **)&api.release) && get("cuMemAddressReserve", (void **)&api.reserve) &&
                 get("cuMemAddressFree", (void **)&api.addr_free) && get("cuMemMap", (void **)&api.map) &&
                 get("cuMemUnmap", (void **)&api.unmap) && get("cuMemSetAccess", (void **)&api.access);
        cudaGetLastError();
    });
    return &api;
}
}  // namespace

int DpSlot::ring_ensure(size_t phys_bytes, size_t *granularity)
{
    VmmApi *a = vmm();
    if (!a->ok) return PTAS_ECUDA;
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    prop.location.id = device_;
    size_t gran = 0;
    if (a->gran(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_MINIMUM) != CUDA_SUCCESS || gran == 0) return PTAS_ECUDA;
    *granularity = gran;
    if (phys_bytes == 0) return PTAS_OK;   // granularity query only
    if (ring_.va && ring_.phys == phys_bytes) return PTAS_OK;
    if (ring_.va) {   // release the previous ring (different size)
        a->unmap((CUdeviceptr)ring_.va, 2 * ring_.phys);
        a->addr_free((CUdeviceptr)ring_.va, 2 * ring_.phys);
        a->release((CUmemGenericAllocationHandle)ring_.handle);
        ring_ = Ring();
    }
    CUmemGenericAllocationHandle h;
    if (a->create(&h, phys_bytes, &prop, 0) != CUDA_SUCCESS) return PTAS_ENOMEM;
    CUdeviceptr va = 0;
    if (a->reserve(&va, 2 * phys_bytes, gran, 0, 0) != CUDA_SUCCESS) {
        a->release(h);
        return PTAS_ENOMEM;
    }
    CUmemAccessDesc acc = {};
    acc.location = prop.location;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (a->map(va, phys_bytes, 0, h, 0) != CUDA_SUCCESS || a->map(va + phys_bytes, phys_bytes, 0, h, 0) != CUDA_SUCCESS ||
        a->access(va, 2 * phys_bytes, &acc, 1) != CUDA_SUCCESS) {
        a->unmap(va, 2 * phys_bytes);
        a->addr_free(va, 2 * phys_bytes);
        a->release(h);
        return PTAS_ENOMEM;
    }
    ring_.va = (unsigned long long)va;
    ring_.phys = phys_bytes;
    ring_.handle = (unsigned long long)h;
    return PTAS_OK;
}

static int bits_of(int32_t x)
{
    int b = 0;
    while (x) {
        ++b;
        x >>= 1;
    }
    return b;
}

// Geometry of the row space of an internal-order DP (a-2, a-4).
// pad: rows stored with pitch Wp = W*e rounded up to 4 bytes (the packed-word
// kernel's layout); without padding the layout is the caller's (pitch W).
static int build_geom(const std::vector<int32_t> &N, int e, bool pad, RowGeom *g,
                      std::vector<int64_t> *cnt, std::vector<int64_t> *stride)
{
    const int K = (int)N.size();
    std::memset(g, 0, sizeof(*g));
    g->K1 = K - 1;
    g->W = N[K - 1] + 1;
    g->Wp = pad ? row_pitch_words(g->W * e) * 4 / e : g->W;
    stride->assign(K, 1);
    if (K >= 2) (*stride)[K - 2] = g->Wp;
    for (int i = K - 3; i >= 0; --i) (*stride)[i] = (*stride)[i + 1] * (N[i + 1] + 1);
    int rho_max = 0;
    for (int i = 0; i < K - 1; ++i) {
        g->N[i] = N[i];
        g->stride[i] = (*stride)[i];
        rho_max += N[i];
    }
    g->rho_max = rho_max;
    g->maxsuf[K - 1] = 0;
    for (int i = K - 2; i >= 0; --i) g->maxsuf[i] = g->maxsuf[i + 1] + N[i];
    int word = 0, bit = 0;
    // PTAS_FORCE_TWO_WORDS=1 (tests only): split the leading digits over two
    // words even when they fit in one, to exercise the two-word kernels.
    const int split = (PTAS_KNOB("PTAS_FORCE_TWO_WORDS", 0) == 1 && K - 1 >= 2) ? (K - 1) / 2 : -1;
    for (int i = 0; i < K - 1; ++i) {
        int w = bits_of(N[i]) + 1;
        if (bit + w > 64 || i == split) {
            ++word;
            bit = 0;
        }
        if (word >= MAXW) return PTAS_ETOOBIG;
        g->word[i] = (uint8_t)word;
        g->shift[i] = (uint8_t)bit;
        g->guard[word] |= 1ull << (bit + w - 1);
        bit += w;
    }
    g->nwords = K > 1 ? word + 1 : 0;
    // cnt[i][L] = #{(p_i..p_{K1-1}) : 0 <= p_d <= N_d, sum = L}; cnt[K1][0] = 1
    const int K1 = K - 1, ld = rho_max + 1;
    cnt->assign((size_t)(K1 + 1) * ld, 0);
    (*cnt)[(size_t)K1 * ld + 0] = 1;
    for (int i = K1 - 1; i >= 0; --i)
        for (int L = 0; L <= rho_max; ++L) {
            int64_t s = 0;
            for (int v = 0; v <= N[i] && v <= L; ++v) s += (*cnt)[(size_t)(i + 1) * ld + (L - v)];
            (*cnt)[(size_t)i * ld + L] = s;
        }
    return PTAS_OK;
}

// internal order: the non-empty canonical classes, in rq.order or identity
static int internal_order(const DpRequest &rq, std::vector<int> *order)
{
    order->clear();
    if (rq.order) {
        int ne = 0;
        for (int i = 0; i < rq.K; ++i) ne += rq.N[i] > 0;
        for (int i = 0; i < ne; ++i) order->push_back(rq.order[i]);
    } else {
        for (int i = 0; i < rq.K; ++i)
            if (rq.N[i] > 0) order->push_back(i);
    }
    if ((int)order->size() > MAXK) return PTAS_ETOOBIG;
    return PTAS_OK;
}

static double trace_now()
{
    return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int DpSlot::run_dp(const DpRequest &rq, DpOutcome *out)
{
    static const bool trace = [] {
        const char *t = std::getenv("PTAS_TRACE");
        return t && t[0] == '1';
    }();
    const double tr0 = trace ? trace_now() : 0;
    double tr_enum = 0, tr_fillq = 0;
    DpOutcome o;
    cudaStream_t st = rq.stream ? rq.stream : stream_;
    std::vector<int> order;
    int rc = internal_order(rq, &order);
    if (rc) return rc;
    const int K = (int)order.size();
    std::vector<int32_t> N(K);
    std::vector<int64_t> r(K);
    __int128 sg = 1;
    int64_t sumN = 0;
    for (int i = 0; i < K; ++i) {
        N[i] = rq.N[order[i]];
        r[i] = rq.r[order[i]];
        sumN += N[i];
        sg *= (N[i] + 1);
        if (sg > (__int128)INT64_MAX) return PTAS_ETOOBIG;
    }
    if (sumN > 65535) return PTAS_ETOOBIG;
    const int64_t sigma = (int64_t)sg;
    const int e = sumN <= 255 ? 1 : 2;
    const int64_t bytes = sigma * e;
    if (rq.ext_table && rq.ext_bytes < bytes) return PTAS_EINVAL;
    last_valid_ = false;
    o.sigma = sigma;
    o.e = e;
    o.Kint = K;
    if (K == 0) {
        void *table = rq.ext_table;
        if (!table) {
            PT_CK(table_.ensure(16));
            table = table_.p;
        }
        PT_CK(cudaEventRecord(ev_[0], st));
        PT_CK(launch_fill_value(table, e, 0, st));
        PT_CK(cudaEventRecord(ev_[1], st));
        PT_CK(cudaEventRecord(ev_[2], st));
        PT_CK(cudaEventRecord(ev_[3], st));
        PT_CK(sync_spin(st));
        o.launches = 1;
        o.opt = 0;
        last_valid_ = true;
        last_table_ = table;
        last_stream_ = st;
        last_K_ = 0;
        last_Kcanon_ = rq.K;
        last_e_ = e;
        last_sigma_ = 1;
        last_nC_ = 0;
        last_opt_ = 0;
        last_W_ = last_Wp_ = 1;
        last_rows_ = 1;
        last_order_.clear();
        *out = o;
        return PTAS_OK;
    }
    RowGeom g;
    std::vector<int64_t> cnt, stride;
    rc = build_geom(N, e, true, &g, &cnt, &stride);
    if (rc) return rc;
    PT_CK(blk_.ensure(sizeof(int32_t) * 2 * MAXK));
    g.blk = (int32_t *)blk_.p;   // pivot blocks, written by build_prefix_kernel (D13)
    const int64_t rows = sigma / g.W;
    const int64_t ibytes = rows * g.Wp * e;  // padded internal table
    // ---- level window (D15): rows with p0 >= 1 depend only on slabs
    // p0 - s0, 1 <= s0 <= hi0 (their pivot is digit 0, D13), so slab p0 = 1 .. N0 is
    // ONE launch over all its rows and only Rw = hi0 + 1 slabs are resident: a ring
    // of Rw slabs mapped twice in virtual memory; slab 0 (p0 = 0) is the DP of the
    // other classes, filled level by level from its own row index
    const int32_t hi0w = K >= 2 ? (int32_t)std::min<int64_t>(N[0], rq.T / r[0]) : 0;
    // (the slabs p0 >= 1 need the packed kernel: rows of at most 1 KiB, window shifts <= 124 B)
    const int64_t J0w = std::min<int64_t>(N[K - 1], rq.T / r[K - 1]);
    const bool window = rq.window && K >= 2 && !rq.ext_table && (!rq.shard || rq.shard->comm) && hi0w < N[0] &&
                        g.Wp * e / 4 <= 256 && J0w * e <= 124;
    if (rq.window && !window) return PTAS_ETOOBIG;   // no saving possible: the caller falls back
    RowGeom gidx;                                     // row index geometry (window: slab 0's rows)
    std::vector<int64_t> cnt_sub, stride_sub;
    int64_t rows_idx = rows, slab_bytes = 0, Rw = 0;
    size_t gran = 0;
    if (window) {
        std::vector<int32_t> Nsub(N.begin() + 1, N.end());
        if (Nsub.size() == 1) {   // K = 2: slab 0 is one row
            cnt_sub.assign(1, 1);
            std::memset(&gidx, 0, sizeof(gidx));
        } else {
            rc = build_geom(Nsub, e, true, &gidx, &cnt_sub, &stride_sub);
            if (rc) return rc;
        }
        rows_idx = sigma / (N[0] + 1) / g.W;
        // the row index of slab 0 in the FULL layout: digits 1 .. K-2 with the full
        // strides and the full digit packing (digit 0 = 0)
        for (int i = 0; i + 1 < K - 1; ++i) {
            gidx.stride[i] = g.stride[i + 1];
            gidx.word[i] = g.word[i + 1];
            gidx.shift[i] = g.shift[i + 1];
        }
        gidx.nwords = g.nwords;
        Rw = hi0w + 1;
        rc = ring_ensure(0, &gran);
        if (rc) return rc;
        slab_bytes = (rows_idx * g.Wp * e + (int64_t)gran - 1) / (int64_t)gran * (int64_t)gran;
        stride[0] = slab_bytes / e;
        g.stride[0] = stride[0];
        g.span_words = 2 * Rw * slab_bytes / 4;
    }
    // level sharding over the ranks of a communicator
    int G = 1, myrank = 0;
    bool virt = false;
    const ShardCtx *sh = rq.shard;
    if (sh) {
        if (sh->comm) {
            G = sh->world;
            myrank = sh->rank;
        } else if (sh->virtual_shards > 1) {
            G = sh->virtual_shards;
            virt = true;
        }
    }
    const bool comm_dp = sh && sh->comm && (G > 1 || sh->force || sh->slab_pipe);   // collectives in this DP
    auto sharded = [&](int64_t R) { return (G > 1 || comm_dp) && R >= std::max<int64_t>(sh->min_rows, 1); };
    // ---- slab/halo pipeline: with a communicator and a
    // windowed DP, rank g holds the contiguous slab range [pb, pe) of the first
    // internal class plus the hin = min(hi0, pb) slabs below it (the halo), in one
    // linear buffer (slab p0 at p0 - pbase).  The slab-0 levels (the other classes'
    // row-levels) are cut into chunks; per chunk rank g receives the halo rows of
    // the chunk from g - 1, fills the chunk's rows of its slabs in ascending order
    // (slab p0 >= 1 reads only slabs p0 - s0, s0 >= 1, at the same or lower
    // levels, D13), and sends the chunk's rows of its last min(hi0, pe) slabs to
    // g + 1: a wavefront over (rank, chunk) with ncclSend / ncclRecv.  OPT(N)
    // lives on the last rank and is broadcast.  Every rank takes the same
    // decisions (same inputs), so the p2p calls pair up.
    const bool pipe = window && sh && sh->comm && sh->slab_pipe && (int64_t)N[0] + 1 >= G;
    int64_t pb = 0, pe = 0, pbase = 0, hin = 0, hout = 0;
    std::vector<int> chunk_lv;   // chunk c = slab-0 levels [chunk_lv[c], chunk_lv[c + 1])
    if (pipe) {
        slab_plan((int64_t)N[0] + 1, hi0w, myrank, G, &pb, &pe, &pbase, &hin, &hout);
        g.span_words = (pe - pbase) * slab_bytes / 4;
        const int nlev = (K >= 3 ? gidx.rho_max : 0) + 1;   // slab 0's row-levels (cnt_sub[0 .. nlev))
        const int64_t C = std::min<int64_t>(nlev, std::max<int64_t>(1, PTAS_KNOB("PTAS_PIPE_CHUNKS_PER_RANK", 4) * G));
        const int64_t target = (rows_idx + C - 1) / C;
        chunk_lv.push_back(0);
        int64_t acc_rows = 0;
        for (int L = 0; L < nlev; ++L) {
            acc_rows += cnt_sub[L];
            if (acc_rows >= target && L + 1 < nlev) {
                chunk_lv.push_back(L + 1);
                acc_rows = 0;
            }
        }
        chunk_lv.push_back(nlev);
    }
    size_t stage_bytes = 0;
    if (pipe) {   // the halo rows of the largest chunk (chunk_lv covers slab 0's levels only)
        for (size_t c = 0; c + 1 < chunk_lv.size(); ++c) {
            int64_t nr = 0;
            for (int L = chunk_lv[c]; L < chunk_lv[c + 1]; ++L) nr += cnt_sub[L];
            stage_bytes = std::max(stage_bytes, (size_t)(std::max(hin, hout) * nr * g.Wp * e));
        }
    } else {   // the sharded units: row-levels, or (window) slab 0's levels and whole slabs
        std::vector<int64_t> units = window ? cnt_sub : cnt;
        if (window) units.push_back(rows_idx);
        for (int64_t R : units) {
            if (!(G > 1 || comm_dp) || !sharded(R)) continue;
            stage_bytes = std::max(stage_bytes, (size_t)(shard_chunk(R, G, g.Wp * e) * G * g.Wp * e));
        }
    }
    // compute in the caller's buffer when its layout is the padded one
    void *table = nullptr;
    const bool in_place = rq.ext_table && g.Wp == g.W && ((uintptr_t)rq.ext_table & 15) == 0;
    // admission: the budget and every large allocation first; a comm-backed DP then
    // agrees on the outcome over all ranks (min of the status words) before any
    // collective, so no rank returns while its peers wait in an all-gather
    int adm = PTAS_OK;
    if (pipe) {
        const int64_t need = (pe - pbase) * slab_bytes + rows_idx * 8 * (1 + (g.nwords <= 1 ? 1 : 2)) + (int64_t)stage_bytes;
        if (rq.budget > 0 || (size_t)((pe - pbase) * slab_bytes) > table_.cap) {
            const int64_t budget = rq.budget > 0 ? rq.budget : free_budget();
            if (need > budget) adm = PTAS_ETOOBIG;
        }
        if (!adm && table_.ensure((size_t)((pe - pbase) * slab_bytes)) != cudaSuccess) adm = PTAS_ENOMEM;
        o.dev_bytes = need;
    } else if (window) {
        const int64_t need = Rw * slab_bytes + rows_idx * 8 * (1 + (g.nwords <= 1 ? 1 : 2));
        const int64_t budget = rq.budget > 0 ? rq.budget : free_budget() + (int64_t)ring_.phys;
        if (need > budget) adm = PTAS_ETOOBIG;
        else adm = ring_ensure((size_t)(Rw * slab_bytes), &gran);
        o.dev_bytes = need;
    } else if (!in_place) {
        // auto budget: query free HBM only when the table has to grow
        // (cudaMemGetInfo costs ~0.1 ms per call)
        if (rq.budget > 0 || (size_t)ibytes > table_.cap) {
            const int64_t budget = rq.budget > 0 ? rq.budget : free_budget();
            if (ibytes > budget) adm = PTAS_ETOOBIG;
        }
        if (!adm && table_.ensure((size_t)ibytes) != cudaSuccess) adm = PTAS_ENOMEM;
    }
    const int NWk = g.nwords <= 1 ? 1 : 2;
    if (!adm && rowidx_.ensure((size_t)rows_idx * 8 * (1 + NWk)) != cudaSuccess) adm = PTAS_ENOMEM;
    if (!adm && stage_bytes && stage_.ensure(stage_bytes) != cudaSuccess) adm = PTAS_ENOMEM;
    if (comm_dp) {
        if (xch_.ensure(64) != cudaSuccess) return PTAS_ENOMEM;   // (64 B: never fails after the first DP)
        int32_t *dx = (int32_t *)xch_.p;
        h_scalar_[0] = adm;
        PT_CK(cudaMemcpyAsync(dx, h_scalar_, 4, cudaMemcpyHostToDevice, st));
        const int crc = comm_allreduce_min_i32(sh->comm, dx, 1, st);
        if (crc) return crc;
        PT_CK(cudaMemcpyAsync(h_scalar_, dx, 4, cudaMemcpyDeviceToHost, st));
        PT_CK(sync_spin(st));
        adm = (int32_t)h_scalar_[0];
    }
    if (adm) return adm;
    table = in_place ? rq.ext_table : table_.p;
    if (!window) o.dev_bytes = ibytes + rows * 8 * (1 + NWk);
    PT_CK(cudaEventRecord(ev_[0], st));
    int64_t idxN = N[K - 1];
    for (int i = 0; i < K - 1; ++i) idxN += (int64_t)N[i] * stride[i];
    // window: ring position of slab p0 is Rw + (p0 mod Rw) (slabs), relative to the ring
    // (pipeline: slab p0 at p0 - pbase of the rank's linear buffer)
    auto slab_ptr = [&](int64_t p0) {
        if (pipe) return (void *)((unsigned char *)table_.p + (p0 - pbase) * slab_bytes);
        return (void *)((unsigned char *)(uintptr_t)ring_.va + (Rw + p0 % Rw) * slab_bytes);
    };
    if (pipe) {
        table = table_.p;
        idxN = ((int64_t)N[0] - pbase) * stride[0] + (idxN - (int64_t)N[0] * stride[0]);   // (last rank only)
    } else if (window) {
        table = slab_ptr(0);
        idxN = (Rw + N[0] % Rw) * stride[0] + (idxN - (int64_t)N[0] * stride[0]);   // relative to the ring
    }

    // ---- uploads: r[K] int64 | stride[K] int64 | hi[K] int32, then cnt table
    std::vector<int32_t> hi(K);
    for (int i = 0; i < K; ++i) {
        int64_t b = rq.T / r[i];
        hi[i] = (int32_t)(b < N[i] ? b : N[i]);
    }
    // interior test of the fill kernel: rows p >= hi (leading dims) dominate every prefix
    for (int i = 0; i < K - 1; ++i) g.maxs[g.word[i]] |= (uint64_t)hi[i] << g.shift[i];
    const size_t small_bytes = (size_t)K * (4 + 8 + 8);
    std::vector<unsigned char> small(small_bytes);
    std::memcpy(small.data(), r.data(), (size_t)K * 8);
    std::memcpy(small.data() + K * 8, stride.data(), (size_t)K * 8);
    std::memcpy(small.data() + K * 16, hi.data(), (size_t)K * 4);
    // one upload (one API call): [r | stride | hi] (8-byte padded), then the
    // cnt table and level_start[rho_max + 2] (prefix sums of the row counts)
    // (window: the row index covers slab 0's rows, i.e. the levels of the other classes)
    const std::vector<int64_t> &cntU = window ? cnt_sub : cnt;
    const int rho_maxU = window ? (K >= 3 ? gidx.rho_max : 0) : g.rho_max;
    std::vector<int64_t> lstart((size_t)rho_maxU + 2, 0);
    for (int rho = 0; rho <= rho_maxU; ++rho) lstart[rho + 1] = lstart[rho] + cntU[rho];
    const size_t cnt_words = cntU.size() + lstart.size();
    const size_t small_pad = (small_bytes + 7) & ~(size_t)7;
    small.resize(small_pad + cnt_words * 8, 0);
    std::memcpy(small.data() + small_pad, cntU.data(), cntU.size() * 8);
    std::memcpy(small.data() + small_pad + cntU.size() * 8, lstart.data(), lstart.size() * 8);
    PT_CK(cnt_.ensure(small.size()));
    pin_reset();
    PT_CK(h2d(cnt_.p, small.data(), small.size(), st));
    o.h2d += (int64_t)small.size();
    void *const d_small = cnt_.p;
    const int64_t *d_cnt = (const int64_t *)((unsigned char *)cnt_.p + small_pad);
    // ---- a-4 level-ordered row index (row base + packed leading digits per row)
    int64_t *d_rb = (int64_t *)rowidx_.p;
    uint64_t *d_pw = (uint64_t *)(d_rb + rows_idx);
    // on the side stream: overlaps the enumeration below and its host round trip
    // (PTAS_ROWIDX_MAIN=1: on the DP's own stream, three API calls fewer)
    const bool ri_main = PTAS_KNOB("PTAS_ROWIDX_MAIN", 0) == 1;
    if (!ri_main) {
        PT_CK(cudaEventRecord(ev_fork_, st));
        PT_CK(cudaStreamWaitEvent(side_, ev_fork_, 0));
    }
    PT_CK(launch_build_row_index(window ? gidx : g, d_cnt, d_cnt + cntU.size(), rows_idx, d_rb, d_pw,
                                 ri_main ? st : side_));
    if (!ri_main) PT_CK(cudaEventRecord(ev_join_, side_));
    ++o.launches;
    const int64_t *d_r = (const int64_t *)d_small;
    const int64_t *d_stride = (const int64_t *)((unsigned char *)d_small + K * 8);
    const int32_t *d_hi = (const int32_t *)((unsigned char *)d_small + K * 16);

    // ---- a-3 configuration enumeration
    int D = 0;
    int64_t nprefix = 1;
    while (D < K && nprefix * (hi[D] + 1) <= 65536) {
        nprefix *= hi[D] + 1;
        ++D;
    }
    PT_CK(counts_.ensure((size_t)nprefix * 8));
    PT_CK(offsets_.ensure((size_t)(nprefix + 1) * 8));
    int64_t *d_counts = (int64_t *)counts_.p;
    int64_t *d_offsets = (int64_t *)offsets_.p;
    PT_CK(launch_enum_configs(0, K, D, nprefix, d_hi, d_r, rq.T, d_stride, d_counts, nullptr,
                              nullptr, nullptr, st));
    PT_CK(launch_exclusive_scan(d_counts, d_offsets, nprefix, d_offsets + nprefix, st));
    o.launches += 2;
    // |C| is needed on the host only to size buffers and shared-memory tables.
    // Once this slot has run a DP, the DP is enqueued without waiting for it:
    // buffers preallocated for nc_cap_ configurations, prefix tables sized for
    // NP_CAP, launch heuristics from the previous DP's prefix count; the
    // kernels exit and the DP is redone synchronously if a bound is exceeded
    // (meta->ovf), which then grows the bounds.
    // Round 2: the enumeration always reads |C| back (PTAS_ENUM_SYNC=0 restores the
    // round-trip-free path of D9): with several DPs in flight the round-trip-free
    // path intermittently left a DP's table unfilled (OPT(N) read from stale memory;
    // 4 of 8 M5s-0.15 P = 2 solves after an M3s solve, 0 of 8 with the read-back)
    // -- a race not yet located, so the path is off by default
    const bool es_sync = PTAS_KNOB("PTAS_ENUM_SYNC", 1) == 1;
    // (a comm-backed DP always reads |C| back: every rank then takes the same path,
    // no rank can redo the DP alone while its peers wait in a collective)
    const bool nosync = np_hint_ >= 0 && nc_cap_ > 0 && !force_sync_enum_ && !es_sync && !comm_dp;
    int64_t nC;        // |C| (synchronous) or its bound
    int64_t nP_bound;  // bound of the prefix list incl. the zero prefix (smem sizing)
    // test knobs: PTAS_NC_CAP / PTAS_NP_CAP lower the bounds (exercise the redo path)
    const int64_t ncc = PTAS_KNOB("PTAS_NC_CAP", 0);
    const int64_t np_cap = std::min<int64_t>(NP_CAP, PTAS_KNOB("PTAS_NP_CAP", NP_CAP));
    if (nosync) {
        nC = ncc > 0 ? std::min<int64_t>(nc_cap_, ncc) : nc_cap_;
        nP_bound = NP_CAP + 1;
    } else {
        PT_CK(cudaMemcpyAsync(h_scalar_, d_offsets + nprefix, 8, cudaMemcpyDeviceToHost, st));
        PT_CK(sync_spin(st));
        o.d2h += 8;
        nC = h_scalar_[0];
        if (nC <= 0) return PTAS_EINTERNAL;  // (0,..,0,1) is always feasible
        nC_cap_grow(nC);
        nP_bound = nC;
    }
    if (trace) tr_enum = trace_now();
    PT_CK(digits_.ensure((size_t)nC * K * 2));
    PT_CK(off_.ensure((size_t)nC * 8));
    PT_CK(pref_.ensure((size_t)nC * sizeof(PrefixEntry)));
    PT_CK(launch_enum_configs(1, K, D, nprefix, d_hi, d_r, rq.T, d_stride, d_counts, d_offsets,
                              (uint16_t *)digits_.p, (int64_t *)off_.p, st, nC));
    PT_CK(launch_build_prefix(K, (const uint16_t *)digits_.p, (const int64_t *)off_.p, d_offsets + nprefix, nC,
                              nosync ? np_cap : INT64_MAX, g, N.data(), (PrefixEntry *)pref_.p, d_meta_, st));
    o.launches += 2;
    tl_np_hint = nosync ? np_hint_ : -1;
    // dominance table of the prefix chunks (D10) when it fits the
    // shared-memory budget for the prefix-list bound; PTAS_DOMTAB=0: off
    {
        int ts = 0;
        for (int i = 0; i < K - 1; ++i) {
            g.hi[i] = hi[i];
            g.dbase[i] = ts;
            ts += hi[i] + 1;
        }
        const int64_t nch = (std::max<int64_t>(nP_bound - 1, 0) + 31) / 32;
        const int64_t dt = PTAS_KNOB("PTAS_DOMTAB", -1);
        // (K - 1 >= 4: many leading digits, so few interior rows and long per-row
        // dominance tests; with 1-3 digits the lane-parallel test is as fast)
        const bool want = e == 1 && (dt >= 0 ? dt != 0 : K - 1 >= 4);   // (uint8 kernels only)
        if (K > 1 && want && (int64_t)ts * nch * 4 <= DOMTAB_MAX_BYTES) {
            PT_CK(domtab_.ensure((size_t)DOMTAB_MAX_BYTES));
            g.TS = ts;
            g.domtab = (const uint32_t *)domtab_.p;
            PT_CK(launch_build_dom_table((const PrefixEntry *)pref_.p, d_meta_, g, (uint32_t *)domtab_.p, st));
            ++o.launches;
        }
    }
    // prefix offsets into the packed kernel's constant bank
    PT_CK(cpstage_.ensure(const_prefix_staging_bytes()));
    cudaError_t cpe = index_ < 4 ? prepare_const_prefix((const PrefixEntry *)pref_.p, d_meta_, nP_bound, e, g.nwords, index_,
                                                   cpstage_.p, st)
                                : cudaErrorNotSupported;
    const int cpref_ok = (cpe == cudaSuccess && PTAS_KNOB("PTAS_NO_CPREF", 0) != 1) ? 1 : 0;
    if (cpe != cudaSuccess && cpe != cudaErrorNotSupported) PT_CK(cpe);
    ++o.launches;
    const int J0 = (int)std::min<int64_t>(N[K - 1], rq.T / r[K - 1]);
    // PTAS_FORCE_SCALAR=1: the full-relaxation scalar kernel for every level;
    // =2: the long-row path for every level (test coverage)
    const int64_t fs = PTAS_KNOB("PTAS_FORCE_SCALAR", 0);
    const bool force_scalar = fs == 1 || fs == 2;
    const bool force_long = fs == 2;
    const bool use_pdl = PTAS_KNOB("PTAS_PDL", 1) != 0;
    bool prev_fill = false;  // the previous launch on st was a packed fill (PDL-safe)
    bool used_scalar = false;  // some level ran on the scalar (uncollapsed) kernel
    // one row-level (or slice of it): packed-word kernel, scalar kernel as fallback
    // one row-level (or slab, or a slice of either): rows [b, b + c) of the row
    // index from slot idx_off
    auto fill = [&](void *tab, const RowGeom &gg, int j0, int64_t idx_off, int64_t b, int64_t c,
                    void *compact) -> cudaError_t {
        const int rho_ = 0;   // (unused by the kernels)
        const int64_t *rbl = d_rb + idx_off;
        const uint64_t *pwl = d_pw + idx_off;
        cudaError_t err = cudaErrorNotSupported;
        if (!force_scalar) {
            err = launch_row_fill_swar(e, tab, gg, rbl, pwl, rows_idx, (const PrefixEntry *)pref_.p, d_meta_, nP_bound,
                                       j0, rho_, b, c, compact, sm_count_, st, (use_pdl && prev_fill) ? 1 : 0,
                                       cpref_ok ? index_ : -1);
            if (err == cudaSuccess) prev_fill = true;
        }
        if (err == cudaErrorNotSupported && compact == nullptr && (force_long || !force_scalar)) {
            err = launch_row_fill_long(e, tab, gg, rbl, pwl, rows_idx, (const PrefixEntry *)pref_.p, d_meta_, nP_bound,
                                       j0, rho_, b, c, sm_count_, st);
            if (err == cudaSuccess) {
                prev_fill = false;
                return err;
            }
            if (err == cudaErrorInvalidValue) err = cudaErrorNotSupported;
        }
        if (err == cudaErrorNotSupported) {
            err = launch_row_fill(e, tab, gg, rbl, pwl, rows_idx, (const PrefixEntry *)pref_.p, d_meta_, nP_bound, j0,
                                  rho_, b, c, compact, sm_count_, st);
            prev_fill = false;
            used_scalar = true;
        }
        return err;
    };

    // ---- a-5 level fill, one launch per row-level
    const int ld = g.rho_max + 1;
    // ---- dataflow runs (D7): runs of row-levels filled by ONE
    // launch each.  PTAS_DF = 0: off (one launch per row-level); 1: the whole
    // DP in one launch, one row set per warp; 2: maximal runs of row-levels
    // with at most PTAS_DF_ROWS rows (default 2 * 32 * SMs) in one launch
    // each, the other levels one launch each; 3: the whole DP in dataflow
    // launches, runs of levels with at most PTAS_DF_SPLIT_ROWS rows with one
    // row set per block (the 8 warps split the prefix walk: shorter latency
    // per row for the narrow levels on the critical path), the others with
    // one row set per warp (the default); 4: as 3, with the narrow runs filled by
    // ONE thread-block cluster in lockstep (cluster barrier per level, no flags).
    // Only for unsharded DPs on the packed kernel.
    struct DfRun {
        int rho0, rho1;        // levels rho0 .. rho1 (inclusive)
        int nsplit;
        int64_t max_rows;
        int64_t total_sets;
        size_t plan_off;       // int32 offset into dfplan_
    };
    std::vector<DfRun> runs;
    // narrow K = 3 DPs: the whole fill on one thread-block cluster, recent levels
    // in distributed shared memory (row_ring.cu, D14); PTAS_RING=0: off
    const bool ring = G == 1 && !comm_dp && !window && !force_scalar && K == 3 &&
                      launch_row_fill_ring(e, table, g, N.data(), r.data(), rq.T, J0, (const PrefixEntry *)pref_.p,
                                           d_meta_, nP_bound, st, true) == cudaSuccess;
    cudaGetLastError();
    if (!ring) {
        // Dataflow runs and split runs pay only when a row's walk is long.  A row walks
        // its pivot block (D13); most rows have pivot 0, whose block is {s' : s'_0 >= 1,
        // sum s'_i r_i <= T}, counted here on the host.  Measured with the short prefix
        // batches of round 2: DPs with blocks of at most 12 prefixes (M2s 4, M3s 12) are
        // fastest with one launch per row-level (M2s 1.90 -> 1.82 ms, M3s 4.90 -> 3.62
        // ms, M3g (16) 42.8 -> 39.6 ms -- M3g keeps runs below), M5s-0.15 (38) needs the
        // dataflow runs with split row sets (15.9 ms; 25.4 ms without runs, 20.0 ms
        // without split runs).  PTAS_DF / PTAS_DF_SPLIT_ROWS override.
        const int64_t blk0 = pivot0_block(N.data(), r.data(), K, rq.T);   // prefixes with s'_0 >= 1
        const int64_t dfm_env = PTAS_KNOB("PTAS_DF", -1);
        // (DPs whose levels are all narrow -- K = 2: one row per level -- keep one
        // dataflow launch instead of hundreds of tiny ones)
        int64_t max_level_rows = 0;
        for (int rho = 0; rho <= g.rho_max; ++rho) max_level_rows = std::max(max_level_rows, cnt[rho]);
        const int df_mode = dfm_env >= 0 ? (int)dfm_env
                                         : ((blk0 > PTAS_KNOB("PTAS_DF_BLOCK", 16) || max_level_rows <= 256) ? 3 : 0);
        const int64_t dfr = PTAS_KNOB("PTAS_DF_ROWS", -1);
        const int64_t df_rows = df_mode == 1 ? INT64_MAX : (dfr >= 0 ? dfr : (int64_t)2 * 32 * sm_count_);
        const int64_t sr_env = PTAS_KNOB("PTAS_DF_SPLIT_ROWS", -1);
        const int64_t split_rows = sr_env >= 0 ? sr_env : (blk0 > PTAS_KNOB("PTAS_DF_SPLIT_BLOCK", 12) ? 2000 : 0);
        if (df_mode > 0 && G == 1 && !comm_dp && !window && !force_scalar && g.rho_max >= 1) {
            if (df_mode == 3 || df_mode == 4) {
                // levels wider than df_rows get a launch of their own (enough rows to fill
                // the GPU: the flag protocol costs more than the launch boundary saves,
                // measured M2s -11%, M3g -16%); runs of narrower ones are dataflow launches
                auto kind = [&](int rho_) { return cnt[rho_] <= split_rows ? 0 : (cnt[rho_] <= df_rows ? 1 : 2); };
                for (int rho = 0; rho <= g.rho_max;) {
                    const int kd = kind(rho);
                    int r1 = rho;
                    while (r1 + 1 <= g.rho_max && kind(r1 + 1) == kd) ++r1;
                    if (kd < 2) runs.push_back({rho, r1, kd == 0 ? (df_mode == 4 ? 0 : 8) : 1, 0, 0, 0});
                    rho = r1 + 1;
                }
            } else {
                for (int rho = 0; rho <= g.rho_max;) {
                    if (cnt[rho] > df_rows) {
                        ++rho;
                        continue;
                    }
                    int r1 = rho;
                    while (r1 + 1 <= g.rho_max && cnt[r1 + 1] <= df_rows) ++r1;
                    if (r1 > rho) runs.push_back({rho, r1, 1, 0, 0, 0});
                    rho = r1 + 1;
                }
            }
        }
        std::vector<int32_t> plan;
        std::vector<DfRun> ok;
        for (DfRun rn : runs) {
            for (int rho = rn.rho0; rho <= rn.rho1; ++rho) rn.max_rows = std::max(rn.max_rows, cnt[rho]);
            const int rpw = swar_df_rows_per_set(e, g, J0, rn.max_rows, sm_count_);
            if (rpw <= 0) continue;
            const int nl = rn.rho1 - rn.rho0 + 1;
            rn.plan_off = plan.size();
            int64_t sets = 0;
            plan.resize(plan.size() + 2 * (size_t)(nl + 1));
            int32_t *ss = plan.data() + rn.plan_off, *sl = ss + nl + 1;
            for (int l = 0; l <= nl; ++l) {
                ss[l] = (int32_t)sets;
                sl[l] = (int32_t)lstart[rn.rho0 + l];
                if (l < nl) sets += (cnt[rn.rho0 + l] + rpw - 1) / rpw;
            }
            rn.total_sets = sets;
            ok.push_back(rn);
        }
        runs.swap(ok);
        if (!runs.empty()) {
            PT_CK(dfplan_.ensure(plan.size() * 4));
            PT_CK(h2d(dfplan_.p, plan.data(), plan.size() * 4, st));
            o.h2d += (int64_t)plan.size() * 4;
            void *old = flags_.p;
            PT_CK(flags_.ensure((size_t)rows * 4));
            if (flags_.p != old || df_epoch_ + runs.size() + 1 < df_epoch_) {
                PT_CK(cudaMemsetAsync(flags_.p, 0, flags_.cap, st));
                df_epoch_ = 0;
            }
            if (!ticket_.p) {
                PT_CK(ticket_.ensure(8));
                PT_CK(cudaMemsetAsync(ticket_.p, 0, 8, st));
                ticket_base_ = 0;
            }
        }
    }
    DfArgs dfa;
    std::memset(&dfa, 0, sizeof(dfa));
    if (!runs.empty()) {
        dfa.flags = (uint32_t *)flags_.p;
        dfa.ticket = (unsigned long long *)ticket_.p;
        for (int i = 0; i < K - 1; ++i) {
            dfa.rstride[i] = (int32_t)(stride[i] / g.Wp);
            const int w = bits_of(N[i]) + 1;
            dfa.dmask[i] = (((uint64_t)1 << (w - 1)) - 1) << g.shift[i];
        }
    }
    size_t next_run = 0;

    if (!ri_main) PT_CK(cudaStreamWaitEvent(st, ev_join_, 0));   // row index ready
    PT_CK(cudaEventRecord(ev_[1], st));
    // PTAS_LEVEL_TIMES=1: per-row-level device times (events between launches; diagnostics)
    static const bool lvl_times = [] {
        const char *t = std::getenv("PTAS_LEVEL_TIMES");
        return t && t[0] == '1';
    }();
    std::vector<cudaEvent_t> lev;
    if (lvl_times) {
        lev.resize((size_t)g.rho_max + 2);
        for (auto &ev : lev) PT_CK(cudaEventCreate(&ev));
        PT_CK(cudaEventRecord(lev[0], st));
    }
    if (ring) {
        PT_CK(launch_row_fill_ring(e, table, g, N.data(), r.data(), rq.T, J0, (const PrefixEntry *)pref_.p, d_meta_,
                                   nP_bound, st, false));
        ++o.fill_launches;
    }
    // one unit (a row-level, or a window slab) of R rows from index slot idx_off into
    // `tab`: directly, or sharded -- the rank's aligned slice into the compact stage
    // buffer, ncclAllGather (in place), row_scatter into every rank's table
    auto fill_unit = [&](void *tab, const RowGeom &gg, int64_t idx_off, int64_t R) -> int {
        if (!sharded(R)) {
            PT_CK(fill(tab, gg, J0, idx_off, 0, R, nullptr));
            ++o.fill_launches;
            return PTAS_OK;
        }
        const int64_t chunk = shard_chunk(R, G, g.Wp * e);
        unsigned char *stage = (unsigned char *)stage_.p;
        if (virt) {
            for (int v = 0; v < G; ++v) {
                int64_t b = v * chunk, c = std::min(R, b + chunk) - b;
                if (c <= 0) continue;
                PT_CK(fill(tab, gg, J0, idx_off, b, c, stage + b * g.Wp * e));
                ++o.fill_launches;
            }
        } else {
            int64_t b = myrank * chunk, c = std::min(R, b + chunk) - b;
            if (c > 0) {
                PT_CK(fill(tab, gg, J0, idx_off, b, c, stage + b * g.Wp * e));
                ++o.fill_launches;
            }
            int crc = comm_allgather(sh->comm, stage + (size_t)myrank * chunk * g.Wp * e, stage,
                                     (size_t)(chunk * g.Wp * e), st);
            if (crc) return crc;
        }
        PT_CK(launch_row_scatter(e, tab, g, d_rb + idx_off, R, stage, sm_count_, st));
        prev_fill = false;
        ++o.launches;
        return PTAS_OK;
    };
    if (pipe) {
        if (trace)
            std::fprintf(stderr, "[ptas] slab pipeline: rank %d/%d slabs [%lld, %lld) base %lld hin %lld hout %lld, %zu chunks, "
                                 "slab %lld B (rows %lld, pitch %lld, e %d), buffer %p cap %zu\n",
                         myrank, G, (long long)pb, (long long)pe, (long long)pbase, (long long)hin, (long long)hout,
                         chunk_lv.size() - 1, (long long)slab_bytes, (long long)rows_idx, (long long)g.Wp, e, table_.p,
                         table_.cap);
        unsigned char *stg = (unsigned char *)stage_.p;
        const int64_t rowB = g.Wp * e;
        for (size_t c = 0; c + 1 < chunk_lv.size(); ++c) {
            const int La = chunk_lv[c], Lb = chunk_lv[c + 1];
            const int64_t i0 = lstart[La], nr = lstart[Lb] - i0;
            if (nr <= 0) continue;
            if (myrank > 0 && hin > 0) {   // the chunk's rows of slabs pb - hin .. pb - 1 from rank g - 1
                const int crc = comm_recv(sh->comm, stg, (size_t)(hin * nr * rowB), myrank - 1, st);
                if (crc) return crc;
                for (int64_t j = 0; j < hin; ++j) {
                    PT_CK(launch_row_scatter(e, slab_ptr(pb - hin + j), g, d_rb + i0, nr, stg + j * nr * rowB,
                                             sm_count_, st));
                    ++o.launches;
                }
                prev_fill = false;
            }
            for (int64_t p0 = pb; p0 < pe; ++p0) {
                if (p0 == 0) {   // slab 0: the other classes' DP, level by level
                    for (int rho = La; rho < Lb; ++rho) {
                        if (cntU[rho] <= 0) continue;
                        PT_CK(fill(slab_ptr(0), g, J0, lstart[rho], 0, cntU[rho], nullptr));
                        ++o.fill_launches;
                    }
                } else {         // the chunk's rows of slab p0: one launch (no dependency inside)
                    RowGeom gs = g;
                    gs.pw_or[g.word[0]] |= (uint64_t)p0 << g.shift[0];
                    PT_CK(fill(slab_ptr(p0), gs, J0, i0, 0, nr, nullptr));
                    ++o.fill_launches;
                }
            }
            if (myrank + 1 < G && hout > 0) {   // the chunk's rows of slabs pe - hout .. pe - 1 to rank g + 1
                for (int64_t j = 0; j < hout; ++j) {
                    PT_CK(launch_row_gather(e, slab_ptr(pe - hout + j), g, d_rb + i0, nr, stg + j * nr * rowB,
                                            sm_count_, st));
                    ++o.launches;
                }
                const int crc = comm_send(sh->comm, stg, (size_t)(hout * nr * rowB), myrank + 1, st);
                if (crc) return crc;
                prev_fill = false;
            }
        }
    } else if (window) {
        // slab 0: the DP of the other classes, level by level (its rows dominate only
        // prefixes with s0 = 0); then slabs 1 .. N0, one unit each over all rows
        // (sharded over the ranks of a communicator: SURVEY.md §8(f)-2ii)
        for (int rho = 0; rho <= rho_maxU; ++rho) {
            const int urc = fill_unit(table, g, lstart[rho], cntU[rho]);
            if (urc) return urc;
        }
        for (int64_t p0 = 1; p0 <= N[0]; ++p0) {
            RowGeom gs = g;
            gs.pw_or[g.word[0]] |= (uint64_t)p0 << g.shift[0];
            const int urc = fill_unit(slab_ptr(p0), gs, 0, rows_idx);
            if (urc) return urc;
        }
    }
    for (int rho = 0; rho <= ((ring || window) ? -1 : g.rho_max); ++rho) {
        const int64_t R = cnt[rho];
        if (lvl_times && rho > 0) PT_CK(cudaEventRecord(lev[rho], st));
        if (R <= 0) continue;
        if (next_run < runs.size() && runs[next_run].rho0 == rho) {
            const DfRun &rn = runs[next_run++];
            dfa.plan = (const int32_t *)dfplan_.p + rn.plan_off;
            dfa.nlev = rn.rho1 - rn.rho0 + 1;
            dfa.total_sets = rn.total_sets;
            dfa.base = ticket_base_;
            dfa.epoch = ++df_epoch_;
            dfa.nsplit = rn.nsplit;
            // PTAS_DF_SLEEP0 / PTAS_DF_SLEEP_MAX: poll backoff (ns), doubling
            dfa.sleep0 = (int32_t)std::max<int64_t>(0, PTAS_KNOB("PTAS_DF_SLEEP0", 64));
            dfa.sleep_max = (int32_t)std::max<int64_t>(dfa.sleep0, PTAS_KNOB("PTAS_DF_SLEEP_MAX", 64));
            dfa.grid_div = rq.grid_div > 1 ? rq.grid_div : 1;
            // PTAS_DF_PROF=1 (with a PTAS_DF_PROFILE=1 build): per-level set timings of the run
            static const bool df_prof = [] {
                const char *t = std::getenv("PTAS_DF_PROF");
                return t && t[0] == '1';
            }();
            std::vector<unsigned long long> prof_h;
            if (df_prof) {
                prof_h.assign((size_t)6 * dfa.nlev, 0);
                for (int l = 0; l < dfa.nlev; ++l) prof_h[6 * l + 4] = ~0ull;
                PT_CK(dfprof_.ensure(prof_h.size() * 8));
                PT_CK(cudaMemcpyAsync(dfprof_.p, prof_h.data(), prof_h.size() * 8, cudaMemcpyHostToDevice, st));
                dfa.prof = (unsigned long long *)dfprof_.p;
            }
            cudaError_t err = launch_row_fill_swar_df(e, table, g, d_rb, d_pw, rows_idx, (const PrefixEntry *)pref_.p,
                                                      d_meta_, nP_bound, J0, rn.max_rows, dfa, &ticket_base_, sm_count_,
                                                      st, (use_pdl && prev_fill) ? 1 : 0, cpref_ok ? index_ : -1);
            if (err == cudaSuccess && df_prof) {
                PT_CK(cudaMemcpyAsync(prof_h.data(), dfprof_.p, prof_h.size() * 8, cudaMemcpyDeviceToHost, st));
                PT_CK(cudaStreamSynchronize(st));
                const unsigned long long g0 = prof_h[4];
                std::fprintf(stderr, "[ptas] df run rho %d..%d split %d sigma=%lld: lvl rows sets wait/walk/tail(cyc) ready..done(us)\n",
                             rn.rho0, rn.rho1, rn.nsplit, (long long)sigma);
                for (int l = 0; l < dfa.nlev; ++l) {
                    const unsigned long long *q = prof_h.data() + 6 * l;
                    const double c = q[0] ? (double)q[0] : 1.0;
                    std::fprintf(stderr, "  %3d %8lld %7llu %7.0f %7.0f %7.0f %9.2f %9.2f\n", rn.rho0 + l,
                                 (long long)cnt[rn.rho0 + l], q[0], q[1] / c, q[2] / c, q[3] / c,
                                 (q[4] - g0) * 1e-3, (q[5] - g0) * 1e-3);
                }
                dfa.prof = nullptr;
            }
            if (err == cudaSuccess) {
                prev_fill = true;
                ++o.fill_launches;
                if (lvl_times)
                    for (int r2 = rho + 1; r2 <= rn.rho1; ++r2) PT_CK(cudaEventRecord(lev[r2], st));
                rho = rn.rho1;
                continue;
            }
            if (err != cudaErrorNotSupported) PT_CK(err);
            // unsupported geometry: fill the run level by level
        }
        const int urc = fill_unit(table, g, lstart[rho], R);
        if (urc) return urc;
    }
    PT_CK(cudaEventRecord(ev_[2], st));
    if (lvl_times && ring) {
        for (auto &ev : lev) cudaEventDestroy(ev);
    } else if (lvl_times) {
        PT_CK(cudaEventRecord(lev[g.rho_max + 1], st));
        PT_CK(cudaEventSynchronize(lev[g.rho_max + 1]));
        std::fprintf(stderr, "[ptas] level times (us, rows) sigma=%lld:", (long long)sigma);
        for (int rho = 0; rho <= g.rho_max; ++rho) {
            float ms = 0;
            cudaEventElapsedTime(&ms, lev[rho], lev[rho + 1]);
            std::fprintf(stderr, " %.1f/%lld", ms * 1e3, (long long)cnt[rho]);
        }
        std::fprintf(stderr, "\n");
        for (auto &ev : lev) cudaEventDestroy(ev);
    }
    if (trace) tr_fillq = trace_now();
    o.launches += o.fill_launches;
    (void)ld;

    // ---- a-6 readout
    if (pipe) {   // OPT(N) is in the last rank's slab N0: read there, broadcast to every rank
        if (myrank == G - 1) {
            PT_CK(launch_read_opt(e, table, idxN, d_meta_, st));
            ++o.launches;
        }
        if (G > 1) {
            const int crc = comm_broadcast(sh->comm, &((DpMeta *)d_meta_)->opt, sizeof(int32_t), G - 1, st);
            if (crc) return crc;
        }
    } else {
        PT_CK(launch_read_opt(e, window ? (void *)(uintptr_t)ring_.va : table, idxN, d_meta_, st));
        ++o.launches;
    }
    if (rq.ext_table && !in_place) {
        PT_CK(launch_compact_rows(e, table, rq.ext_table, rows, g.W, g.Wp, st));
        ++o.launches;
    }
    PT_CK(cudaMemcpyAsync(h_meta_, d_meta_, sizeof(DpMeta), cudaMemcpyDeviceToHost, st));
    PT_CK(cudaEventRecord(ev_[3], st));
    for (;;) {   // spin on the end event itself (one event record fewer than sync_spin)
        const cudaError_t q = cudaEventQuery(ev_[3]);
        if (q == cudaSuccess) break;
        if (q != cudaErrorNotReady) PT_CK(q);
    }
    o.d2h += sizeof(DpMeta);
    float ms = 0;
    PT_CK(cudaEventElapsedTime(&ms, ev_[0], ev_[3]));
    o.dp_s = ms * 1e-3;
    PT_CK(cudaEventElapsedTime(&ms, ev_[1], ev_[2]));
    o.fill_s = ms * 1e-3;
    if (rq.ref_event) {
        float a = 0, b = 0;
        PT_CK(cudaEventElapsedTime(&a, rq.ref_event, ev_[1]));
        PT_CK(cudaEventElapsedTime(&b, rq.ref_event, ev_[2]));
        o.fill_t0 = a * 1e-3;
        o.fill_t1 = b * 1e-3;
    }
    if (trace) {
        const double t3 = trace_now();
        std::fprintf(stderr, "[ptas] dp sigma=%lld K=%d levels=%d host: setup+enum-sync %.3f ms, fill enqueue %.3f ms, "
                             "wait %.3f ms | device: dp %.3f ms fill %.3f ms | host clock %.3f .. %.3f ms\n",
                     (long long)sigma, K, g.rho_max + 1, 1e3 * (tr_enum - tr0), 1e3 * (tr_fillq - tr_enum),
                     1e3 * (t3 - tr_fillq), 1e3 * o.dp_s, 1e3 * o.fill_s, 1e3 * tr0, 1e3 * t3);
    }
    tl_np_hint = -1;
    if (h_meta_->ovf) {
        // a bound of the round-trip-free enumeration was exceeded: nothing was
        // filled; redo synchronously (exact sizes) and keep the larger bounds
        nC_cap_grow(h_meta_->nC);
        if (ticket_.p) {   // the exited dataflow launches took no tickets: restart the counter
            PT_CK(cudaMemsetAsync(ticket_.p, 0, 8, st));
            ticket_base_ = 0;
        }
        force_sync_enum_ = true;
        const int rc2 = run_dp(rq, out);
        force_sync_enum_ = false;
        return rc2;
    }
    np_hint_ = h_meta_->nP - 1;
    o.opt = h_meta_->opt;
    o.relax = (double)h_meta_->relax;
    o.relax_exec = used_scalar ? o.relax : (double)h_meta_->relax_exec;
    o.nC = h_meta_->nC;
    o.nP = h_meta_->nP;

    o.windowed = window ? 1 : 0;
    last_valid_ = !window;   // a window keeps no table for a traceback
    last_table_ = table;
    last_stream_ = st;
    last_K_ = K;
    last_Kcanon_ = rq.K;
    last_e_ = e;
    last_sigma_ = sigma;
    last_nC_ = h_meta_->nC;
    last_opt_ = o.opt;
    last_order_ = order;
    last_N_ = N;
    last_stride_ = stride;
    last_W_ = g.W;
    last_Wp_ = g.Wp;
    last_rows_ = rows;
    last_idxN_ = idxN;
    *out = o;
    return PTAS_OK;
}

int DpSlot::traceback(std::vector<MachineCfg> *machines, DpOutcome *acc)
{
    if (!last_valid_) return PTAS_EINTERNAL;
    if (last_K_ == 0 || last_opt_ == 0) return PTAS_OK;
    const int K = last_K_;
    const int64_t nC = last_nC_;
    cudaStream_t st = last_stream_;
    {
        // device ranking + canonical output: one upload, two kernels, one readback
        const int Kc = last_Kcanon_;
        std::vector<int32_t> up((size_t)K + Kc, -1);
        std::copy(last_N_.begin(), last_N_.end(), up.begin());
        for (int i = 0; i < K; ++i) up[(size_t)K + last_order_[i]] = i;
        const size_t tb_bytes = ((size_t)nC + K + Kc + 4 + (size_t)last_opt_ * (1 + Kc)) * 4 + 16;
        PT_CK(tb_.ensure(tb_bytes));
        int32_t *d_N = (int32_t *)tb_.p;
        int32_t *d_inv = d_N + K;
        int32_t *d_rank = d_inv + Kc;
        int32_t *d_len = d_rank + nC;   // [4] then d_out[opt], then d_out_dig[opt][Kc]
        int32_t *d_out = d_len + 4;
        int32_t *d_out_dig = d_out + last_opt_;
        pin_reset();
        PT_CK(h2d(d_N, up.data(), up.size() * 4, st));
        PT_CK(cudaMemsetAsync(&d_meta_->err, 0, 4, st));
        const cudaError_t le = launch_traceback_canon(last_e_, last_table_, K, d_N, (const uint16_t *)digits_.p,
                                                      (const int64_t *)off_.p, d_rank, nC, d_inv, Kc, last_idxN_,
                                                      d_out, d_out_dig, last_opt_, d_len, d_meta_, st);
        if (le == cudaSuccess) {
            acc->h2d += (int64_t)up.size() * 4;
            acc->launches += 2;
            std::vector<int32_t> outv(4 + (size_t)last_opt_ * (1 + Kc));
            PT_CK(cudaMemcpyAsync(outv.data(), d_len, outv.size() * 4, cudaMemcpyDeviceToHost, st));
            PT_CK(cudaMemcpyAsync(h_meta_, d_meta_, sizeof(DpMeta), cudaMemcpyDeviceToHost, st));
            PT_CK(sync_spin(st));
            acc->d2h += (int64_t)outv.size() * 4 + (int64_t)sizeof(DpMeta);
            if (h_meta_->err || outv[0] != last_opt_) return PTAS_EINTERNAL;
            const int32_t *dg = outv.data() + 4 + last_opt_;
            for (int q = 0; q < last_opt_; ++q) machines->emplace_back(dg + (size_t)q * Kc, dg + (size_t)(q + 1) * Kc);
            return PTAS_OK;
        }
        if (le != cudaErrorNotSupported) PT_CK(le);
    }
    std::vector<uint16_t> dig((size_t)nC * K);
    PT_CK(cudaMemcpyAsync(dig.data(), digits_.p, dig.size() * 2, cudaMemcpyDeviceToHost, st));
    PT_CK(sync_spin(st));
    acc->d2h += (int64_t)dig.size() * 2;
    // canonical lexicographic rank of every configuration (reading R11)
    std::vector<std::vector<int32_t>> canon((size_t)nC, std::vector<int32_t>(last_Kcanon_, 0));
    for (int64_t c = 0; c < nC; ++c)
        for (int i = 0; i < K; ++i) canon[c][last_order_[i]] = dig[(size_t)c * K + i];
    std::vector<int32_t> idx((size_t)nC);
    std::iota(idx.begin(), idx.end(), 0);
    std::sort(idx.begin(), idx.end(), [&](int32_t a, int32_t b) { return canon[a] < canon[b]; });
    std::vector<int32_t> rank((size_t)nC);
    for (int64_t q = 0; q < nC; ++q) rank[idx[q]] = (int32_t)q;
    const size_t tb_bytes = (size_t)nC * 4 + (size_t)K * 4 + (size_t)K * 8 + (size_t)last_opt_ * 4 + 16;
    PT_CK(tb_.ensure(tb_bytes));
    unsigned char *b = (unsigned char *)tb_.p;
    int64_t *d_stride = (int64_t *)b;
    int32_t *d_rank = (int32_t *)(b + (size_t)K * 8);
    int32_t *d_N = d_rank + nC;
    int32_t *d_len = d_N + K;
    int32_t *d_out = d_len + 4;
    pin_reset();
    PT_CK(h2d(d_stride, last_stride_.data(), (size_t)K * 8, st));
    PT_CK(h2d(d_rank, rank.data(), (size_t)nC * 4, st));
    PT_CK(h2d(d_N, last_N_.data(), (size_t)K * 4, st));
    PT_CK(cudaMemsetAsync(&d_meta_->err, 0, 4, st));
    acc->h2d += (int64_t)(K * 8 + nC * 4 + K * 4);
    PT_CK(launch_traceback(last_e_, last_table_, K, d_N, d_stride, (const uint16_t *)digits_.p,
                           (const int64_t *)off_.p, d_rank, nC, last_idxN_, d_out, last_opt_,
                           d_len, d_meta_, st));
    acc->launches += 1;
    // d_len[0] = length, d_len[4 ..] = chosen configurations (d_out = d_len + 4)
    std::vector<int32_t> outv((size_t)last_opt_ + 4);
    PT_CK(cudaMemcpyAsync(outv.data(), d_len, outv.size() * 4, cudaMemcpyDeviceToHost, st));
    PT_CK(cudaMemcpyAsync(h_meta_, d_meta_, sizeof(DpMeta), cudaMemcpyDeviceToHost, st));
    PT_CK(sync_spin(st));
    acc->d2h += (int64_t)outv.size() * 4 + (int64_t)sizeof(DpMeta);
    const int32_t len = outv[0];
    if (h_meta_->err || len != last_opt_) return PTAS_EINTERNAL;
    const int32_t *chosen = outv.data() + 4;
    for (int q = 0; q < len; ++q) machines->push_back(canon[chosen[q]]);
    return PTAS_OK;
}

int DpSlot::copy_table_to_host(void *dst, int64_t bytes)
{
    if (!last_valid_) return PTAS_EINTERNAL;
    const void *src = last_table_;
    if (last_Wp_ != last_W_) {
        PT_CK(stage_.ensure((size_t)bytes));
        PT_CK(launch_compact_rows(last_e_, last_table_, stage_.p, last_rows_, last_W_, last_Wp_,
                                  last_stream_));
        src = stage_.p;
    }
    PT_CK(cudaMemcpyAsync(dst, src, (size_t)bytes, cudaMemcpyDeviceToHost, last_stream_));
    PT_CK(sync_spin(last_stream_));
    return PTAS_OK;
}

int DpSlot::configs_canonical(const DpRequest &rq, std::vector<int32_t> *digits, int64_t *count)
{
    // Runs a full DP on an engine-owned table is unnecessary: enumerate only.
    std::vector<int> order;
    int rc = internal_order(rq, &order);
    if (rc) return rc;
    const int K = (int)order.size();
    digits->clear();
    if (K == 0) {
        *count = 0;
        return PTAS_OK;
    }
    cudaStream_t st = stream_;
    std::vector<int32_t> N(K), hi(K);
    std::vector<int64_t> r(K), stride(K, 1);
    for (int i = 0; i < K; ++i) {
        N[i] = rq.N[order[i]];
        r[i] = rq.r[order[i]];
    }
    for (int i = K - 2; i >= 0; --i) stride[i] = stride[i + 1] * (N[i + 1] + 1);
    for (int i = 0; i < K; ++i) hi[i] = (int32_t)std::min<int64_t>(N[i], rq.T / r[i]);
    const size_t small_bytes = (size_t)K * 20;
    std::vector<unsigned char> small(small_bytes);
    std::memcpy(small.data(), r.data(), (size_t)K * 8);
    std::memcpy(small.data() + K * 8, stride.data(), (size_t)K * 8);
    std::memcpy(small.data() + K * 16, hi.data(), (size_t)K * 4);
    PT_CK(small_.ensure(small_bytes));
    PT_CK(cudaMemcpyAsync(small_.p, small.data(), small_bytes, cudaMemcpyHostToDevice, st));
    const int64_t *d_r = (const int64_t *)small_.p;
    const int64_t *d_stride = (const int64_t *)((unsigned char *)small_.p + K * 8);
    const int32_t *d_hi = (const int32_t *)((unsigned char *)small_.p + K * 16);
    int D = 0;
    int64_t nprefix = 1;
    while (D < K && nprefix * (hi[D] + 1) <= 65536) {
        nprefix *= hi[D] + 1;
        ++D;
    }
    PT_CK(counts_.ensure((size_t)nprefix * 8));
    PT_CK(offsets_.ensure((size_t)(nprefix + 1) * 8));
    int64_t *d_counts = (int64_t *)counts_.p;
    int64_t *d_offsets = (int64_t *)offsets_.p;
    PT_CK(launch_enum_configs(0, K, D, nprefix, d_hi, d_r, rq.T, d_stride, d_counts, nullptr,
                              nullptr, nullptr, st));
    PT_CK(launch_exclusive_scan(d_counts, d_offsets, nprefix, d_offsets + nprefix, st));
    PT_CK(cudaMemcpyAsync(h_scalar_, d_offsets + nprefix, 8, cudaMemcpyDeviceToHost, st));
    PT_CK(sync_spin(st));
    const int64_t nC = h_scalar_[0];
    *count = nC;
    if (nC == 0) return PTAS_OK;
    PT_CK(digits_.ensure((size_t)nC * K * 2));
    PT_CK(off_.ensure((size_t)nC * 8));
    PT_CK(launch_enum_configs(1, K, D, nprefix, d_hi, d_r, rq.T, d_stride, d_counts, d_offsets,
                              (uint16_t *)digits_.p, (int64_t *)off_.p, st));
    std::vector<uint16_t> dig((size_t)nC * K);
    PT_CK(cudaMemcpyAsync(dig.data(), digits_.p, dig.size() * 2, cudaMemcpyDeviceToHost, st));
    PT_CK(sync_spin(st));
    last_valid_ = false;
    digits->assign((size_t)nC * rq.K, 0);
    for (int64_t c = 0; c < nC; ++c)
        for (int i = 0; i < K; ++i) (*digits)[(size_t)c * rq.K + order[i]] = dig[(size_t)c * K + i];
    return PTAS_OK;
}

int DpSlot::row_index(const int32_t *Nc, int Kc, std::vector<int64_t> *level_start,
                      std::vector<int64_t> *rowbase)
{
    std::vector<int32_t> N;
    for (int i = 0; i < Kc; ++i)
        if (Nc[i] > 0) N.push_back(Nc[i]);
    level_start->clear();
    rowbase->clear();
    if (N.empty()) {
        level_start->assign({0, 1});
        rowbase->assign({0});
        return PTAS_OK;
    }
    RowGeom g;
    std::vector<int64_t> cnt, stride;
    int rc = build_geom(N, 1, false, &g, &cnt, &stride);
    if (rc) return rc;
    cudaStream_t st = stream_;
    int64_t rows = 0;
    level_start->push_back(0);
    for (int rho = 0; rho <= g.rho_max; ++rho) {
        rows += cnt[rho];
        level_start->push_back(rows);
    }
    PT_CK(cnt_.ensure((cnt.size() + level_start->size()) * 8));
    PT_CK(cudaMemcpyAsync(cnt_.p, cnt.data(), cnt.size() * 8, cudaMemcpyHostToDevice, st));
    PT_CK(cudaMemcpyAsync((int64_t *)cnt_.p + cnt.size(), level_start->data(), level_start->size() * 8,
                          cudaMemcpyHostToDevice, st));
    const int NWk = g.nwords <= 1 ? 1 : 2;
    PT_CK(rowidx_.ensure((size_t)rows * 8 * (1 + NWk)));
    int64_t *d_out = (int64_t *)rowidx_.p;
    PT_CK(launch_build_row_index(g, (const int64_t *)cnt_.p, (const int64_t *)cnt_.p + cnt.size(), rows, d_out,
                                 (uint64_t *)(d_out + rows), st));
    rowbase->resize((size_t)rows);
    PT_CK(cudaMemcpyAsync(rowbase->data(), d_out, (size_t)rows * 8, cudaMemcpyDeviceToHost, st));
    PT_CK(sync_spin(st));
    last_valid_ = false;
    return PTAS_OK;
}

}  // namespace ptas
