// engine.h — per-device DP engine (host orchestration of the kernels).
#pragma once
#include <algorithm>
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/ptas.h"
#include "internal.h"

namespace ptas {

// How one DP's row-levels are distributed.
struct ShardCtx {
    ptas_comm *comm = nullptr;  // real NCCL ranks (nullptr = none)
    int rank = 0;
    int world = 1;
    int virtual_shards = 1;     // >1: logical shards on this GPU (testing)
    int64_t min_rows = 0;       // row-levels with fewer rows are computed redundantly
    bool force = false;         // shard (slice, all-gather, scatter) also at world size 1
    bool slab_pipe = false;     // windowed DPs: slab/halo pipeline with send/recv
};

struct DpRequest {
    int K = 0;                    // canonical classes (may include zero counts)
    const int32_t *N = nullptr;   // canonical counts
    const int64_t *r = nullptr;   // canonical sizes
    int64_t T = 0;
    const int *order = nullptr;   // internal position i -> canonical class (nullable = identity
                                  // over non-empty classes); must list exactly the non-empty classes
    void *ext_table = nullptr;    // caller device buffer (nullable = engine-owned table)
    int64_t ext_bytes = 0;
    cudaStream_t stream = nullptr;  // nullptr = engine stream
    const ShardCtx *shard = nullptr;
    int64_t budget = 0;           // bytes allowed for the table (0 = auto)
    int window = 0;               // 1: level window (D15): only hi0 + 1 slabs of the
                                  // first internal digit are resident (a ring mapped twice in
                                  // virtual memory); OPT(N) only, no table for a traceback
    int grid_div = 1;             // >1: this many DPs run concurrently; persistent grids take 1/grid_div of the GPU
    cudaEvent_t ref_event = nullptr;  // completed timing event: fill interval reported relative to it
};

struct DpOutcome {
    int32_t opt = 0;
    int64_t sigma = 1;
    int e = 1;
    int Kint = 0;
    double relax = 0;
    double relax_exec = 0;  // relaxations the kernels evaluated (collapsed form, or relax for the scalar kernel)
    int64_t nC = 0, nP = 0;
    double dp_s = 0, fill_s = 0;
    double fill_t0 = -1, fill_t1 = -1;   // fill interval in seconds after rq.ref_event (-1: none)
    int launches = 0, fill_launches = 0;
    int64_t h2d = 0, d2h = 0;
    int windowed = 0;              // the DP ran in level-window mode
    int64_t dev_bytes = 0;         // device memory of its table (ring) and row index
};

// one machine of the traceback: canonical digit vector s (length K canonical)
using MachineCfg = std::vector<int32_t>;

// All per-DP device state: workspace buffers, stream, events, readback
// buffers, and the description of the last DP (for traceback).  Several slots
// run DPs concurrently (one host thread each) for the probes of one round.
class DpSlot {
  public:
    int init(int device, int sm_count, int index);
    int run_dp(const DpRequest &rq, DpOutcome *out);
    // Traceback on the table of the last run_dp (engine-owned or the same
    // ext table); appends OPT(N) canonical configurations to machines.
    int traceback(std::vector<MachineCfg> *machines, DpOutcome *acc);
    // Inspection helpers.
    int configs_canonical(const DpRequest &rq, std::vector<int32_t> *digits, int64_t *count);
    int row_index(const int32_t *N, int K, std::vector<int64_t> *level_start,
                  std::vector<int64_t> *rowbase);
    int64_t free_budget();
    // D2H of the table of the last run_dp (engine-owned or ext).
    int copy_table_to_host(void *dst, int64_t bytes);
    cudaStream_t stream() const { return stream_; }
    bool last_valid() const { return last_valid_; }

    cudaError_t sync_spin(cudaStream_t st);
    // Host<->device copies of small host vectors through a pinned arena (no
    // pageable bounce buffers in the driver); the arena is reset per DP, after
    // the previous DP's final sync.
    cudaError_t h2d(void *dst, const void *src, size_t bytes, cudaStream_t st);
    void pin_reset() { pin_used_ = 0; }

  private:
    struct Buf {
        void *p = nullptr;
        size_t cap = 0;
        cudaError_t ensure(size_t bytes);
    };
    int device_ = -1;
    int sm_count_ = 148;
    int index_ = 0;  // slot index; constant-bank prefix area when < 4
    cudaStream_t stream_ = nullptr;
    cudaEvent_t ev_[4] = {nullptr, nullptr, nullptr, nullptr};
    cudaEvent_t ev_sync_ = nullptr;
    // side stream: the a-4 row index is built concurrently with the a-3
    // enumeration and its host round trip (fork/join events)
    cudaStream_t side_ = nullptr;
    cudaEvent_t ev_fork_ = nullptr, ev_join_ = nullptr;
    DpMeta *d_meta_ = nullptr;
    DpMeta *h_meta_ = nullptr;     // pinned
    // enumeration without a host round trip (D9): configuration
    // buffers preallocated for nc_cap_ configurations; prefix-list length of
    // this slot's last DP (launch heuristics; -1 = none yet: synchronous path)
    int64_t nc_cap_ = 0;
    int64_t np_hint_ = -1;
    bool force_sync_enum_ = false;
    void nC_cap_grow(int64_t nC) { nc_cap_ = std::max<int64_t>(nc_cap_, std::max<int64_t>(4096, 2 * nC)); }
    int64_t *h_scalar_ = nullptr;  // pinned
    unsigned char *pin_ = nullptr;  // pinned arena
    size_t pin_cap_ = 0, pin_used_ = 0;
    Buf table_, digits_, off_, counts_, offsets_, pref_, cnt_, stage_, small_, rank_, tb_, rowidx_, cpstage_;
    // dataflow fill (D7): per-row ready flags, ticket counter, run plans
    Buf flags_, ticket_, dfplan_, dfprof_, domtab_, blk_, xch_;
    // level-window ring (D15): physical slabs mapped twice back to back
    struct Ring {
        unsigned long long va = 0;   // CUdeviceptr of the 2 * phys virtual range
        size_t phys = 0;             // bytes of physical memory (= one mapping)
        unsigned long long handle = 0;
    } ring_;
    int ring_ensure(size_t phys_bytes, size_t *granularity);
    uint32_t df_epoch_ = 0;
    unsigned long long ticket_base_ = 0;

    // state of the last DP (for traceback)
    bool last_valid_ = false;
    void *last_table_ = nullptr;
    cudaStream_t last_stream_ = nullptr;
    int last_K_ = 0, last_Kcanon_ = 0, last_e_ = 1;
    int64_t last_sigma_ = 1, last_nC_ = 0;
    int32_t last_opt_ = 0;
    int64_t last_W_ = 1, last_Wp_ = 1, last_rows_ = 1, last_idxN_ = 0;
    std::vector<int> last_order_;      // internal -> canonical
    std::vector<int32_t> last_N_;      // internal counts
    std::vector<int64_t> last_stride_; // internal strides
};

constexpr int MAX_SLOTS = 12;

// Persistent host workers for the concurrent DPs of one call (speculative chain,
// P probes): creating a std::thread per DP and batch put ~15 us per thread on
// the critical path of every solve (the last DP of an M5s chain was enqueued
// 0.1 ms after the first).  run(n, fn): fn(1 .. n-1) on workers, fn(0) on the
// caller; returns when all n are done.  Workers are never joined (the engine
// lives for the process).
class WorkerPool {
  public:
    void run(int n, const std::function<void(int)> &fn)
    {
        if (n <= 1) {
            if (n == 1) fn(0);
            return;
        }
        {
            std::lock_guard<std::mutex> lk(m_);
            while ((int)th_.size() < n - 1) {
                std::thread t([this] { loop(); });
                t.detach();
                th_.push_back(0);
            }
            job_ = &fn;
            next_ = 1;
            total_ = n;
            remaining_.store(n - 1, std::memory_order_release);
        }
        cv_.notify_all();
        fn(0);
        // the caller's own DP is usually not the last: spin for the others (a
        // condition-variable wake-up costs tens of microseconds on the critical path)
        while (remaining_.load(std::memory_order_acquire) != 0) std::this_thread::yield();
        std::lock_guard<std::mutex> lk(m_);
        job_ = nullptr;
        next_ = total_ = 0;
    }

  private:
    void loop()
    {
        std::unique_lock<std::mutex> lk(m_);
        for (;;) {
            cv_.wait(lk, [&] { return next_ < total_; });
            const int i = next_++;
            const std::function<void(int)> *f = job_;
            lk.unlock();
            (*f)(i);
            remaining_.fetch_sub(1, std::memory_order_acq_rel);
            lk.lock();
        }
    }
    std::mutex m_;
    std::condition_variable cv_;
    std::vector<int> th_;   // one entry per started worker
    const std::function<void(int)> *job_ = nullptr;
    int next_ = 0, total_ = 0;
    std::atomic<int> remaining_{0};
};

// Per-device engine: a lock serialising API calls on the device and up to
// MAX_SLOTS DP slots.  Slot 0 serves every single-DP call.
class Engine {
  public:
    static int get(int device, Engine **out);
    std::mutex mu;
    int device() const { return device_; }
    int sm_count() const { return sm_count_; }
    int slot(int i, DpSlot **out);
    DpSlot *s0() { return slots_[0]; }
    // forwards to slot 0
    int run_dp(const DpRequest &rq, DpOutcome *out) { return slots_[0]->run_dp(rq, out); }
    int traceback(std::vector<MachineCfg> *m, DpOutcome *acc) { return slots_[0]->traceback(m, acc); }
    int configs_canonical(const DpRequest &rq, std::vector<int32_t> *d, int64_t *c)
    {
        return slots_[0]->configs_canonical(rq, d, c);
    }
    int row_index(const int32_t *N, int K, std::vector<int64_t> *ls, std::vector<int64_t> *rb)
    {
        return slots_[0]->row_index(N, K, ls, rb);
    }
    int copy_table_to_host(void *dst, int64_t bytes) { return slots_[0]->copy_table_to_host(dst, bytes); }
    cudaStream_t stream() const { return slots_[0]->stream(); }
    // timing reference of one call: recorded on st and waited for, so the
    // DPs' fill intervals (events on any stream) can be placed on one axis
    int mark_reference(cudaStream_t st, cudaEvent_t *out);
    cudaError_t sync_spin(cudaStream_t st) { return slots_[0]->sync_spin(st); }
    WorkerPool &pool() { return pool_; }
    // device buffer for the multi-GPU exchanges of a solve (grown, never freed)
    int exchange_buffer(size_t bytes, void **out)
    {
        if (bytes > xcap_) {
            if (xbuf_) cudaFree(xbuf_);
            xbuf_ = nullptr;
            xcap_ = 0;
            const size_t want = std::max<size_t>(bytes, 4096);
            if (cudaMalloc(&xbuf_, want) != cudaSuccess) {
                cudaGetLastError();
                return PTAS_ENOMEM;
            }
            xcap_ = want;
        }
        *out = xbuf_;
        return PTAS_OK;
    }

  private:
    WorkerPool pool_;
    void *xbuf_ = nullptr;
    size_t xcap_ = 0;
    int init(int device);
    int device_ = -1;
    int sm_count_ = 148;
    DpSlot *slots_[MAX_SLOTS] = {};
    cudaEvent_t ref_ev_ = nullptr;
};

// NCCL glue (comm.cpp)
int comm_rank(const ptas_comm *c);
int comm_world(const ptas_comm *c);
int comm_allgather(ptas_comm *c, const void *send, void *recv, size_t bytes_per_rank,
                   cudaStream_t st);
int comm_allreduce_min_i32(ptas_comm *c, int32_t *d_buf, size_t count, cudaStream_t st);
int comm_broadcast(ptas_comm *c, void *d_buf, size_t bytes, int root, cudaStream_t st);
int comm_send(ptas_comm *c, const void *d_buf, size_t bytes, int peer, cudaStream_t st);
int comm_recv(ptas_comm *c, void *d_buf, size_t bytes, int peer, cudaStream_t st);

}  // namespace ptas
