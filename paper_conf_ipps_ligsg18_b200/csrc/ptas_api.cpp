// ptas_api.cpp — C ABI entry points and the host driver of the PTAS
// (§8(b)).
//
//   a-1 classify/round            host, O(n log n) per probe
//   a-7 P-probe search + memo     host; DP(T) runs on the GPU (dp_engine.cpp)
//   a-8 schedule at T*            device traceback + host job placement
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <functional>
#include <map>
#include <queue>
#include <thread>
#include <vector>

#include "engine.h"

using namespace ptas;

namespace {

struct Classified {
    int64_t u = 1;
    std::vector<int64_t> r;    // distinct rounded long sizes, ascending
    std::vector<int32_t> N;    // counts
    std::vector<int32_t> cls;  // per job: class or -1
};

int64_t ceil_div(int64_t a, int64_t b) { return a / b + ((a % b) != 0); }

// Alg 1 l.6-8: long iff k*p > T (p > T/k, reading R1);
// u = max(1, floor(T/k^2)) (R2); r = floor(p/u)*u; classes = distinct r
// ascending (R3).
void classify(const int64_t *p, int32_t n, int64_t T, int32_t k, Classified *c)
{
    const int64_t kk = (int64_t)k * k;
    c->u = std::max<int64_t>(1, T / kk);
    const int64_t u = c->u;
    std::vector<int64_t> q;  // rounded multiples floor(p/u) of the long jobs
    q.reserve(n);
    c->cls.assign(n, -1);
    for (int32_t j = 0; j < n; ++j)
        if ((__int128)k * p[j] > (__int128)T) q.push_back(p[j] / u);
    std::sort(q.begin(), q.end());
    q.erase(std::unique(q.begin(), q.end()), q.end());
    c->r.resize(q.size());
    c->N.assign(q.size(), 0);
    for (size_t i = 0; i < q.size(); ++i) c->r[i] = q[i] * u;
    for (int32_t j = 0; j < n; ++j) {
        if (!((__int128)k * p[j] > (__int128)T)) continue;
        int32_t i = (int32_t)(std::lower_bound(q.begin(), q.end(), p[j] / u) - q.begin());
        c->cls[j] = i;
        c->N[i]++;
    }
}

// The same classes and counts (no per-job classes) from the distinct processing
// times and their multiplicities, built once per solve: the search classifies
// every probe (and the speculative chain ahead of it), and with n = 2000 jobs a
// per-job pass costs tens of microseconds per probe on the host's critical path.
struct ValueHistogram {
    std::vector<int64_t> v;    // distinct p, ascending
    std::vector<int32_t> c;    // multiplicities
    ValueHistogram(const int64_t *p, int32_t n)
    {
        if (n <= 0) return;
        int64_t lo = p[0], hi = p[0];
        for (int32_t j = 1; j < n; ++j) {
            lo = std::min(lo, p[j]);
            hi = std::max(hi, p[j]);
        }
        if (hi - lo <= (int64_t)4 * n + 65536) {   // counting (uniform integer sizes: P <= 1000)
            std::vector<int32_t> cnt((size_t)(hi - lo + 1), 0);
            for (int32_t j = 0; j < n; ++j) ++cnt[(size_t)(p[j] - lo)];
            for (size_t i = 0; i < cnt.size(); ++i)
                if (cnt[i]) {
                    v.push_back(lo + (int64_t)i);
                    c.push_back(cnt[i]);
                }
            return;
        }
        std::vector<int64_t> s(p, p + n);
        std::sort(s.begin(), s.end());
        for (int64_t x : s) {
            if (!v.empty() && v.back() == x) ++c.back();
            else {
                v.push_back(x);
                c.push_back(1);
            }
        }
    }
    // classify() with the per-job classes: the class of each distinct long value,
    // then one lookup per job (identical to classify: same r, N, cls)
    void classify_full(const int64_t *p, int32_t n, int64_t T, int32_t k, Classified *out) const
    {
        classify_counts(T, k, out);
        out->cls.assign(n, -1);
        if (out->r.empty()) return;
        const int64_t u = out->u;
        // class index of every distinct value (-1: short)
        std::vector<int32_t> vc(v.size(), -1);
        size_t ci = 0;
        for (size_t i = 0; i < v.size(); ++i) {
            if (!((__int128)k * v[i] > (__int128)T)) continue;
            while (out->r[ci] != (v[i] / u) * u) ++ci;
            vc[i] = (int32_t)ci;
        }
        for (int32_t j = 0; j < n; ++j) {
            const size_t i = (size_t)(std::lower_bound(v.begin(), v.end(), p[j]) - v.begin());
            out->cls[j] = vc[i];
        }
    }
    void classify_counts(int64_t T, int32_t k, Classified *out) const
    {
        const int64_t kk = (int64_t)k * k;
        out->u = std::max<int64_t>(1, T / kk);
        const int64_t u = out->u;
        out->r.clear();
        out->N.clear();
        out->cls.clear();
        // long values: k * p > T, a suffix of the ascending list
        size_t i = (size_t)(std::upper_bound(v.begin(), v.end(), T / k) - v.begin());
        while (i > 0 && (__int128)k * v[i - 1] > (__int128)T) --i;
        while (i < v.size() && !((__int128)k * v[i] > (__int128)T)) ++i;
        for (; i < v.size(); ++i) {
            const int64_t q = v[i] / u;
            if (!out->r.empty() && out->r.back() == q * u) out->N.back() += c[i];
            else {
                out->r.push_back(q * u);
                out->N.push_back(c[i]);
            }
        }
    }
};

int probe_targets(int64_t LB, int64_t UB, int32_t P, std::vector<int64_t> *out)
{
    out->clear();
    if (LB >= UB || P < 1) return PTAS_EINVAL;
    const __int128 w = (__int128)UB - LB;
    for (int32_t j = 0; j < P; ++j) {
        int64_t t = (int64_t)((__int128)LB + ((__int128)(2 * j + 1) * w) / (2 * (__int128)P));
        if (!out->empty() && out->back() == t) continue;
        out->push_back(t);
    }
    return PTAS_OK;
}

// Alg 1 l.10-14 / Alg 3 l.13-25 (reading R8): the smallest feasible probe
// becomes UB; LB rises past every infeasible probe below it.
void interval_update(int64_t *LB, int64_t *UB, const int64_t *T, const int32_t *f, int32_t cnt)
{
    bool any = false;
    int64_t ub = *UB;
    for (int32_t q = 0; q < cnt; ++q)
        if (f[q] && (!any || T[q] < ub)) {
            ub = T[q];
            any = true;
        }
    if (any) {
        int64_t lb = *LB;
        for (int32_t q = 0; q < cnt; ++q)
            if (!f[q] && T[q] < ub) lb = std::max(lb, T[q] + 1);
        *LB = lb;
        *UB = ub;
    } else {
        int64_t mx = *LB;
        for (int32_t q = 0; q < cnt; ++q) mx = std::max(mx, T[q] + 1);
        *LB = mx;
    }
}

int validate_jobs(const int64_t *p, int32_t n, int32_t m, int64_t *LB, int64_t *UB)
{
    if (!p || n < 1 || m < 1) return PTAS_EINVAL;
    __int128 S = 0;
    int64_t mx = 0;
    for (int32_t j = 0; j < n; ++j) {
        if (p[j] < 1) return PTAS_EINVAL;
        S += p[j];
        mx = std::max(mx, p[j]);
    }
    if (S > (__int128)(INT64_MAX / 4)) return PTAS_EINVAL;
    int64_t A = ceil_div((int64_t)S, m);
    *LB = std::max(A, mx);
    *UB = A + mx;
    return PTAS_OK;
}

int k_of(double eps)
{
    if (!(eps > 0.0) || !std::isfinite(eps)) return PTAS_EINVAL;
    double k = std::ceil(1.0 / eps);
    if (!(k >= 1.0) || k > (double)(1 << 20)) return PTAS_EINVAL;
    return (int)k;
}

// memo key: (N, c = r/u, cap = floor(T/u)) — the DP depends only on these
// (sum s_i r_i <= T  <=>  sum s_i c_i <= floor(T/u)), SURVEY.md §8(a) a-7.
std::vector<int64_t> memo_key(const Classified &c, int64_t T)
{
    std::vector<int64_t> key;
    key.reserve(2 * c.N.size() + 2);
    key.push_back((int64_t)c.N.size());
    for (size_t i = 0; i < c.N.size(); ++i) {
        key.push_back(c.N[i]);
        key.push_back(c.r[i] / c.u);
    }
    key.push_back(T / c.u);
    return key;
}

// internal class order for the table (layout 0, D2/D13): the
// non-empty class with the largest count (ties: the highest index) is the
// contiguous row dimension; the leading classes follow by descending size r
// (ties by index), so that the first nonzero leading digit of most rows -- the
// row's pivot, D13 -- is a large class whose block of configurations is short.
// layout 1: the non-empty classes in the given (classify) order.
std::vector<int> choose_order(const std::vector<int32_t> &N, const std::vector<int64_t> &r, int layout)
{
    std::vector<int> o;
    for (size_t i = 0; i < N.size(); ++i)
        if (N[i] > 0) o.push_back((int)i);
    if (layout == 0 && !o.empty()) {
        int last = o[0];
        for (int i : o)
            if (N[i] >= N[last]) last = i;
        std::vector<int> lead;
        for (int i : o)
            if (i != last) lead.push_back(i);
        std::stable_sort(lead.begin(), lead.end(), [&](int a, int b) { return r[a] > r[b]; });
        lead.push_back(last);
        o.swap(lead);
    }
    return o;
}

// internal order for a level-window DP (D15): the row class as in
// layout 0, digit 0 = the class with the most slabs per resident slab,
// (N + 1) / (min(N, T / r) + 1), the other leading classes by descending size
std::vector<int> window_order(const std::vector<int32_t> &N, const std::vector<int64_t> &r, int64_t T)
{
    std::vector<int> o = choose_order(N, r, 0);
    if (o.size() < 3) return o;
    size_t best = 0;
    double bv = -1;
    for (size_t i = 0; i + 1 < o.size(); ++i) {
        const double hi = (double)std::min<int64_t>(N[o[i]], T / r[o[i]]);
        const double v = (N[o[i]] + 1.0) / (hi + 1.0);
        if (v > bv) {
            bv = v;
            best = i;
        }
    }
    std::rotate(o.begin(), o.begin() + best, o.begin() + best + 1);
    return o;
}

double now_s()
{
    return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

struct Acc {
    ptas_stats s;
    std::vector<std::pair<double, double>> iv;   // fill intervals of every DP run (incl. unused speculative ones)
    Acc() { std::memset(&s, 0, sizeof(s)); }
    void interval(const DpOutcome &o)
    {
        if (o.fill_t0 >= 0 && o.fill_t1 > o.fill_t0) iv.emplace_back(o.fill_t0, o.fill_t1);
    }
    // device time during which at least one level-fill loop ran
    void finish_wall()
    {
        std::sort(iv.begin(), iv.end());
        double tot = 0, a = -1, b = -1;
        for (auto &x : iv) {
            if (x.first > b) {
                if (b > a) tot += b - a;
                a = x.first;
                b = x.second;
            } else {
                b = std::max(b, x.second);
            }
        }
        if (b > a) tot += b - a;
        s.fill_wall_seconds = tot;
    }
    void add(const DpOutcome &o)
    {
        interval(o);
        s.relaxations += o.relax;
        s.relax_executed += o.relax_exec;
        s.exec_bytes += (o.relax_exec + (double)o.sigma) * o.e;
        s.dp_seconds += o.dp_s;
        s.fill_seconds += o.fill_s;
        s.alg_bytes += (o.relax + (double)o.sigma) * o.e;
        s.states += o.sigma;
        s.kernel_launches += o.launches;
        s.fill_launches += o.fill_launches;
        s.h2d_bytes += o.h2d;
        s.d2h_bytes += o.d2h;
        s.sigma_max = std::max(s.sigma_max, o.sigma);
        s.window_dps += o.windowed;
        s.dev_bytes_max = std::max(s.dev_bytes_max, o.dev_bytes);
    }
};

int resolve_device(int dev, int *out)
{
    if (dev < 0) {
        if (cudaGetDevice(&dev) != cudaSuccess) {
            cudaGetLastError();
            return PTAS_ECUDA;
        }
    }
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || dev >= n) {
        cudaGetLastError();
        return PTAS_ECUDA;
    }
    if (cudaSetDevice(dev) != cudaSuccess) {
        cudaGetLastError();
        return PTAS_ECUDA;
    }
    *out = dev;
    return PTAS_OK;
}

int solve_core(const int64_t *p, int32_t n, int32_t m, double eps, const ptas_options *opt_in,
               int64_t *makespan_out, int32_t *assignment_out, ptas_stats *stats, ptas_probe *log,
               int32_t log_cap, int32_t *log_len, int64_t extra_h2d, int64_t extra_d2h)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    const double t0 = now_s();
    ptas_options opt;
    ptas_default_options(&opt);
    if (opt_in) opt = *opt_in;
    int64_t LB, UB;
    int rc = validate_jobs(p, n, m, &LB, &UB);
    if (rc) return rc;
    const int k = k_of(eps);
    if (k < 0) return PTAS_EINVAL;
    if (!makespan_out || !assignment_out) return PTAS_EINVAL;
    if (opt.probes_per_round < 1) return PTAS_EINVAL;
    if (opt.mode < PTAS_MODE_SINGLE || opt.mode > PTAS_MODE_MULTI_PROBE) return PTAS_EINVAL;
    if (opt.layout < 0 || opt.layout > 1) return PTAS_EINVAL;
    int rank = 0, world = 1;
    if (opt.comm) {
        rank = comm_rank(opt.comm);
        world = comm_world(opt.comm);
    }
    if (opt.mode == PTAS_MODE_MULTI_PROBE && (!opt.comm || opt.probes_per_round != world))
        return PTAS_EINVAL;
    if (opt.mode == PTAS_MODE_SINGLE && opt.comm) return PTAS_EINVAL;
    const int P = opt.probes_per_round;
    int dev;
    rc = resolve_device(opt.device, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);

    ShardCtx sh;
    const ShardCtx *shp = nullptr;
    if (opt.mode == PTAS_MODE_LEVEL_SHARDED) {
        sh.comm = opt.comm;
        sh.rank = rank;
        sh.world = world;
        sh.virtual_shards = opt.comm ? 1 : std::max(1, opt.virtual_shards);
        sh.min_rows = opt.comm ? (opt.shard_min_rows >= 0 ? opt.shard_min_rows : 2048) : 0;
        sh.force = opt.comm && opt.shard_min_rows == 0;
        sh.slab_pipe = opt.comm && opt.slab_pipeline == 1;
        shp = &sh;
    }

    Acc acc;
    acc.s.h2d_bytes += extra_h2d;
    acc.s.d2h_bytes += extra_d2h;
    cudaEvent_t ref_ev = nullptr;   // time axis of the DPs' fill intervals (fill_wall_seconds)
    {
        const int r2 = eng->mark_reference((cudaStream_t)opt.stream, &ref_ev);
        if (r2) return r2;
    }
    std::map<std::vector<int64_t>, int32_t> memo;
    std::vector<ptas_probe> plog;
    const ValueHistogram hist(p, n);   // classes and counts of every probe (per-job classes: classify)
    if (PTAS_KNOB("PTAS_TRACE", 0) == 1)
        std::fprintf(stderr, "[ptas] histogram built | host clock %.3f .. %.3f ms\n", 1e3 * t0, 1e3 * now_s());
    constexpr int32_t XERR = -1000;                          // MULTI_PROBE: exchanged error codes
    std::vector<std::vector<int64_t>> last_key_of(world);  // MULTI_PROBE: the last DP of each rank
    int round = 0;
    Classified cl;

    // which slot holds the table of which DP key (for the traceback at T*)
    std::vector<std::vector<int64_t>> slot_key(MAX_SLOTS);
    int last_windowed = 0;
    auto make_rq = [&](const Classified &c, int64_t T, const ShardCtx *s, const std::vector<int> &order,
                       cudaStream_t st) {
        DpRequest rq;
        rq.K = (int)c.N.size();
        rq.N = c.N.data();
        rq.r = c.r.data();
        rq.T = T;
        rq.order = order.data();
        rq.shard = s;
        rq.budget = opt.table_budget_bytes;
        rq.stream = st;
        rq.ref_event = ref_ev;
        return rq;
    };
    // One probe DP on a slot; the level window (D15) when options.window
    // asks for it or when the full table does not fit (window = 0), single GPU only
    auto probe_dp = [&](DpSlot *sl, const Classified &c, int64_t T, const ShardCtx *s, cudaStream_t st,
                        int grid_div, DpOutcome *o) -> int {
        // (level-sharded over a communicator too: the slabs are then the sharded units,
        // SURVEY.md §8(f)-2ii; every rank takes the same decision: window = 1, or the
        // ETOOBIG the ranks agreed on at admission)
        const bool can_win = opt.window >= 0 && (!s || s->comm) && opt.mode != PTAS_MODE_MULTI_PROBE;
        std::vector<int> order = choose_order(c.N, c.r, opt.layout);
        DpRequest rq = make_rq(c, T, s, order, st);
        rq.grid_div = grid_div;
        int r2 = PTAS_ETOOBIG;
        if (!(can_win && opt.window == 1)) r2 = sl->run_dp(rq, o);
        if (r2 == PTAS_ETOOBIG && can_win) {
            std::vector<int> worder = window_order(c.N, c.r, T);
            DpRequest rw = make_rq(c, T, s, worder, st);
            rw.grid_div = grid_div;
            rw.window = 1;
            r2 = sl->run_dp(rw, o);
            if (r2 == PTAS_ETOOBIG && opt.window == 1) r2 = sl->run_dp(rq, o);   // no saving possible
        }
        return r2;
    };
    auto run = [&](const Classified &c, int64_t T, const ShardCtx *s, int32_t *opt_out) -> int {
        DpOutcome o;
        int r2 = probe_dp(eng->s0(), c, T, s, (cudaStream_t)opt.stream, 1, &o);
        if (r2) return r2;
        acc.add(o);
        acc.s.unique_dps++;
        *opt_out = o.opt;
        last_windowed = o.windowed;
        return PTAS_OK;
    };
    // Concurrent evaluation of several probes of one round (SINGLE mode): one
    // host thread and one DP slot (own stream and workspace) per probe -- the
    // quarter split of Alg 3 on one GPU.  With a caller
    // stream, slot 0 uses it; the call is host-synchronous either way.
    const bool concurrent = opt.mode == PTAS_MODE_SINGLE && PTAS_KNOB("PTAS_NO_CONCURRENT", 0) != 1;
    // Runs the jobs concurrently (slots 0..), outcomes in outs; grid_div > 0:
    // persistent fill grids take 1/(jobs in flight) of the GPU each.
    auto run_jobs = [&](std::vector<Classified> &cls_v, std::vector<int64_t> &T_v,
                        std::vector<std::vector<int64_t>> &key_v, std::vector<DpOutcome> &outs_all,
                        bool share_grid) -> int {
        const int nj = (int)cls_v.size();
        outs_all.assign(nj, DpOutcome());
        for (int j0 = 0; j0 < nj; j0 += MAX_SLOTS) {
            const int nb = std::min(MAX_SLOTS, nj - j0);
            std::vector<DpSlot *> sl(nb);
            for (int b = 0; b < nb; ++b) {
                int r2 = eng->slot(b, &sl[b]);
                if (r2) return r2;
            }
            std::vector<int> rcs(nb, PTAS_OK);
            std::vector<std::vector<int>> orders(nb);
            for (int b = 0; b < nb; ++b) orders[b] = choose_order(cls_v[j0 + b].N, cls_v[j0 + b].r, opt.layout);
            // persistent fill grids of concurrent DPs: each takes a share of the GPU,
            // 1/nb (PTAS_GRID_SHARE=0) or proportional to its table size (1: the large
            // DPs of a speculative chain outlive the small ones)
            // (PTAS_GRID_DIV=0, experiment: every launch may take the whole GPU)
            std::vector<int> gdiv(nb, 1);
            if (share_grid && PTAS_KNOB("PTAS_GRID_DIV", -1) != 0) {
                const bool prop = PTAS_KNOB("PTAS_GRID_SHARE", 0) == 1;
                std::vector<double> sz(nb, 1.0);
                double tot = 0;
                for (int b = 0; b < nb; ++b) {
                    if (prop)
                        for (int32_t x : cls_v[j0 + b].N) sz[b] *= (double)x + 1.0;
                    tot += sz[b];
                }
                for (int b = 0; b < nb; ++b) gdiv[b] = (int)std::max(1.0, std::min(1e6, std::floor(tot / sz[b])));
            }
            auto work = [&](int b) {
                if (cudaSetDevice(dev) != cudaSuccess) {
                    rcs[b] = PTAS_ECUDA;
                    return;
                }
                rcs[b] = probe_dp(sl[b], cls_v[j0 + b], T_v[j0 + b], nullptr,
                                  b == 0 ? (cudaStream_t)opt.stream : nullptr, gdiv[b], &outs_all[j0 + b]);
            };
            eng->pool().run(nb, work);
            for (int b = 0; b < nb; ++b) {
                if (rcs[b]) return rcs[b];
                slot_key[b] = outs_all[j0 + b].windowed ? std::vector<int64_t>() : key_v[j0 + b];
            }
        }
        return PTAS_OK;
    };
    auto run_many = [&](std::vector<Classified> &cls_v, std::vector<int64_t> &T_v,
                        std::vector<std::vector<int64_t>> &key_v, std::vector<int32_t> &opt_v) -> int {
        const int nj = (int)cls_v.size();
        for (int j0 = 0; j0 < nj; j0 += MAX_SLOTS) {
            const int nb = std::min(MAX_SLOTS, nj - j0);
            std::vector<DpSlot *> sl(nb);
            for (int b = 0; b < nb; ++b) {
                int r2 = eng->slot(b, &sl[b]);
                if (r2) return r2;
            }
            std::vector<DpOutcome> outs(nb);
            std::vector<int> rcs(nb, PTAS_OK);
            std::vector<std::vector<int>> orders(nb);
            for (int b = 0; b < nb; ++b) orders[b] = choose_order(cls_v[j0 + b].N, cls_v[j0 + b].r, opt.layout);
            auto work = [&](int b) {
                if (cudaSetDevice(dev) != cudaSuccess) {
                    rcs[b] = PTAS_ECUDA;
                    return;
                }
                rcs[b] = probe_dp(sl[b], cls_v[j0 + b], T_v[j0 + b], nullptr,
                                  b == 0 ? (cudaStream_t)opt.stream : nullptr, 1, &outs[b]);
            };
            eng->pool().run(nb, work);
            for (int b = 0; b < nb; ++b) {
                if (rcs[b]) return rcs[b];
                acc.add(outs[b]);
                acc.s.unique_dps++;
                opt_v[j0 + b] = outs[b].opt;
                slot_key[b] = outs[b].windowed ? std::vector<int64_t>() : key_v[j0 + b];
            }
        }
        return PTAS_OK;
    };

    // ---- speculative bisection (D8).  With P = 1 the probes are
    // Alg 1's; when the next probe's DP is not known yet, the next `depth`
    // levels of the bisection tree below [LB, UB] (both outcomes of every
    // probe) whose tables are small are evaluated concurrently with it.  A
    // speculative result is used only when Alg 1 actually probes that key,
    // and only then is its work counted; the search itself is unchanged.
    struct SpecRes {
        int32_t opt;
        DpOutcome o;
    };
    std::map<std::vector<int64_t>, SpecRes> spec;
    int spec_depth = opt.speculate < 0 ? 3 : opt.speculate;
    int64_t spec_sigma = (int64_t)1 << 24;
    const bool spec_ring = PTAS_KNOB("PTAS_SPEC_RING", 1) != 0;   // 0: latency-bound DPs only below spec_sigma (A/B)
    const int64_t spec_levels = PTAS_KNOB("PTAS_SPEC_LEVELS", 160);
    const int64_t spec_levels_short = PTAS_KNOB("PTAS_SPEC_LEVELS_SHORT", 480);   // (with a short pivot block)
    const int64_t spec_block = PTAS_KNOB("PTAS_SPEC_BLOCK", 16);
    {
        const int64_t sd = PTAS_KNOB("PTAS_SPEC_DEPTH", -1);
        if (sd >= 0 && opt.speculate < 0) spec_depth = (int)sd;
        const int64_t ss = PTAS_KNOB("PTAS_SPEC_SIGMA", -1);
        if (ss >= 0) spec_sigma = ss;
        if (spec_depth > 3) spec_depth = 3;   // 2^3 - 1 = 7 DPs in flight (MAX_SLOTS slots)
    }
    // Library default (speculate = -1): the feasible-branch chain — the next
    // probes Alg 1 makes if every probe is feasible (the common case: T* = LB,
    // SURVEY §8(d)), 4 deep; all of them are used when the guess holds, none of
    // the tree's other branches occupy the GPU (M2s -5%, M5s-0.2 -44%, measured).
    // speculate = d > 0: the full tree of depth d.  PTAS_SPEC_CHAIN=0 / 1 forces.
    const int64_t sch = PTAS_KNOB("PTAS_SPEC_CHAIN", -1);
    const bool spec_chain = sch >= 0 ? sch == 1 : opt.speculate < 0;
    if (spec_chain && spec_depth > 0)   // (PTAS_SPEC_DEPTH=0 still turns speculation off)
        spec_depth = (int)std::max<int64_t>(1, std::min<int64_t>(MAX_SLOTS, PTAS_KNOB("PTAS_SPEC_CHAIN_DEPTH", 4)));
    const bool spec_on = spec_depth >= 1 && P == 1 && concurrent && opt.memoize && opt.mode == PTAS_MODE_SINGLE;
    auto speculate = [&](int64_t lb0, int64_t ub0) -> int {
        struct Node {
            int64_t lb, ub;
            int d;
        };
        std::vector<Node> q{{lb0, ub0, 0}};
        std::vector<Classified> cls_v;
        std::vector<int64_t> T_v;
        std::vector<std::vector<int64_t>> key_v;
        int depth_lim = spec_depth;
        for (size_t h = 0; h < q.size(); ++h) {
            const Node nd = q[h];
            if (nd.lb >= nd.ub) continue;
            std::vector<int64_t> t1;
            probe_targets(nd.lb, nd.ub, 1, &t1);
            const int64_t T = t1[0];
            Classified c;
            hist.classify_counts(T, k, &c);
            bool take = false, lat = false;
            std::vector<int64_t> key;
            if (!c.N.empty()) {
                key = memo_key(c, T);
                __int128 sg = 1;
                for (int32_t x : c.N) {
                    sg *= (x + 1);
                    if (sg > (__int128)spec_sigma) break;
                }
                const bool known = memo.count(key) || spec.count(key) ||
                                   std::find(key_v.begin(), key_v.end(), key) != key_v.end();
                // latency-bound DPs overlap whatever their size: the K = 3 cluster ring
                // kernel fills them on 16 SMs (D14), and DPs with few wide
                // row-levels (<= spec_levels: the u8 K = 6..8 shapes) leave the GPU idle at
                // every level boundary (measured: M2s -28%, M4s -12%; DPs with hundreds of
                // levels lose by sharing the GPU, M3s +50%)
                if (spec_ring) {
                    const std::vector<int> o = choose_order(c.N, c.r, opt.layout);
                    std::vector<int32_t> No;
                    std::vector<int64_t> ro;
                    for (int i : o) {
                        No.push_back(c.N[i]);
                        ro.push_back(c.r[i]);
                    }
                    lat = ring_fits(No.data(), ro.data(), (int)No.size(), T);
                    int64_t levels = 1;
                    for (size_t i = 0; i + 1 < No.size(); ++i) levels += No[i];
                    lat = lat || (No.size() >= 2 && levels <= spec_levels);
                    // DPs with a few hundred row-levels but short pivot blocks (D13; M3s:
                    // 12 prefixes, 290 levels; M3g: 16, 335) are latency-bound too: their
                    // levels overlap (round 2: M3s 6.3 -> 4.9 ms, M3g 44.9 -> 42.7 ms); with
                    // long blocks (M5s-0.15: 38, 423 levels) they are throughput-bound and
                    // lose by sharing the GPU (15.7 -> 22.1 ms)
                    lat = lat || (No.size() >= 2 && levels <= spec_levels_short &&
                                  pivot0_block(No.data(), ro.data(), (int)No.size(), T, 64) <= spec_block);
                }
                // a large next probe runs alone (throughput-bound: nothing to overlap)
                if (nd.d == 0 && sg > (__int128)spec_sigma && !lat) return PTAS_OK;
                take = !known && (sg <= (__int128)spec_sigma || lat);
            }
            if (take) {
                cls_v.push_back(c);
                T_v.push_back(T);
                key_v.push_back(key);
            }
            // a chain of latency-bound DPs runs deeper: up to MAX_SLOTS DPs over at most
            // 16 probes (memo hits in the chain take no slot), so the whole all-feasible
            // chain of an M5s-shaped search is in flight at once instead of in two batches
            if (lat && spec_chain) depth_lim = (int)PTAS_KNOB("PTAS_SPEC_LAT_DEPTH", 16);
            if (nd.d + 1 < depth_lim && (int)cls_v.size() < MAX_SLOTS) {
                q.push_back({nd.lb, T, nd.d + 1});        // T feasible
                if (!spec_chain) q.push_back({T + 1, nd.ub, nd.d + 1});    // T infeasible
            }
            if ((int)cls_v.size() >= MAX_SLOTS) break;
        }
        if (cls_v.empty()) return PTAS_OK;
        std::vector<DpOutcome> outs;
        if (PTAS_KNOB("PTAS_TRACE", 0) == 1)
            std::fprintf(stderr, "[ptas] speculation planned: %zu DPs | host clock %.3f .. %.3f ms\n", cls_v.size(),
                         1e3 * t0, 1e3 * now_s());
        int r2 = run_jobs(cls_v, T_v, key_v, outs, true);
        if (r2) return r2;
        for (size_t j = 0; j < cls_v.size(); ++j) spec[key_v[j]] = SpecRes{outs[j].opt, outs[j]};
        acc.s.spec_dps += (int32_t)cls_v.size();
        return PTAS_OK;
    };

    while (LB < UB) {
        std::vector<int64_t> Tj;
        probe_targets(LB, UB, P, &Tj);
        if (spec_on) {
            hist.classify_counts(Tj[0], k, &cl);
            if (!cl.N.empty()) {
                const std::vector<int64_t> key = memo_key(cl, Tj[0]);
                if (!memo.count(key) && !spec.count(key)) {
                    rc = speculate(LB, UB);
                    if (rc) return rc;
                }
            }
        }
        const int np = (int)Tj.size();
        std::vector<int32_t> optj(np, 0), hit(np, 0), who(np, 0), Kj(np, 0), xsrc(np, -1);
        std::vector<int64_t> sgj(np, 1);
        std::vector<std::vector<int64_t>> keys(np);
        std::vector<int> pend_q;
        std::vector<Classified> pend_cl;
        std::vector<int64_t> pend_T;
        std::vector<std::vector<int64_t>> pend_key;
        std::vector<std::pair<int, int>> pend_alias;  // probe -> pending job
        for (int q = 0; q < np; ++q) {
            hist.classify_counts(Tj[q], k, &cl);
            Kj[q] = (int32_t)cl.N.size();
            __int128 sg = 1;
            for (int32_t x : cl.N) {
                sg *= (x + 1);
                if (sg > (__int128)INT64_MAX) sg = -1;
                if (sg < 0) break;
            }
            sgj[q] = (int64_t)sg;
            if (cl.N.empty()) {
                optj[q] = 0;
                continue;
            }
            keys[q] = memo_key(cl, Tj[q]);
            auto it = opt.memoize ? memo.find(keys[q]) : memo.end();
            if (it != memo.end()) {
                optj[q] = it->second;
                hit[q] = 1;
                continue;
            }
            auto sp = spec.find(keys[q]);
            if (sp != spec.end()) {   // evaluated speculatively: now it is the search's own DP
                optj[q] = sp->second.opt;
                acc.add(sp->second.o);
                acc.s.unique_dps++;
                memo[keys[q]] = optj[q];
                spec.erase(sp);
                continue;
            }
            // MULTI_PROBE: rank q evaluates probe q, unless an earlier probe of the round
            // has the same DP key (then that rank's result serves both: one DP per key)
            int src = q;
            if (opt.mode == PTAS_MODE_MULTI_PROBE)
                for (int q2 = 0; q2 < q; ++q2)
                    if (keys[q2] == keys[q]) {
                        src = q2;
                        break;
                    }
            xsrc[q] = src;
            const bool mine = opt.mode != PTAS_MODE_MULTI_PROBE || (q == rank && src == q);
            who[q] = opt.mode == PTAS_MODE_MULTI_PROBE ? src : rank;
            if (!mine) {
                optj[q] = -1;  // filled by the exchange
                continue;
            }
            if (concurrent) {
                // deferred: evaluated below with the round's other probes
                bool dup = false;
                for (size_t jj = 0; jj < pend_key.size(); ++jj)
                    if (pend_key[jj] == keys[q]) {
                        pend_alias.push_back({q, (int)jj});
                        dup = true;
                        break;
                    }
                if (!dup) {
                    pend_q.push_back(q);
                    pend_cl.push_back(cl);
                    pend_T.push_back(Tj[q]);
                    pend_key.push_back(keys[q]);
                    pend_alias.push_back({q, (int)pend_key.size() - 1});
                }
                continue;
            }
            rc = run(cl, Tj[q], opt.mode == PTAS_MODE_LEVEL_SHARDED ? shp : nullptr, &optj[q]);
            if (rc && opt.mode == PTAS_MODE_MULTI_PROBE) {
                // every rank must still reach the exchange: the error travels with it
                optj[q] = XERR + rc;
                slot_key[0].clear();
                continue;
            }
            if (rc) return rc;
            slot_key[0] = last_windowed ? std::vector<int64_t>() : keys[q];
            if (opt.memoize) memo[keys[q]] = optj[q];
        }
        if (!pend_q.empty()) {
            std::vector<int32_t> pend_opt(pend_q.size(), 0);
            rc = run_many(pend_cl, pend_T, pend_key, pend_opt);
            if (rc) return rc;
            for (auto &qa : pend_alias) optj[qa.first] = pend_opt[qa.second];
            if (opt.memoize)
                for (size_t jj = 0; jj < pend_key.size(); ++jj) memo[pend_key[jj]] = pend_opt[jj];
        }
        if (opt.mode == PTAS_MODE_MULTI_PROBE) {
            // exchange OPT(N) of every rank's probe (int32 per rank) over NCCL; a
            // failed DP contributes XERR + its status, and then every rank returns it
            std::vector<int32_t> all(world, -1);
            const int32_t mine = rank < np ? optj[rank] : -1;
            int32_t *dbuf = nullptr;
            int xrc = eng->exchange_buffer(sizeof(int32_t) * world, (void **)&dbuf);
            if (xrc) return xrc;
            cudaStream_t st = opt.stream ? (cudaStream_t)opt.stream : eng->stream();
            xrc = eng->s0()->h2d(dbuf + rank, &mine, 4, st) == cudaSuccess ? PTAS_OK : PTAS_ECUDA;
            if (!xrc) xrc = comm_allgather(opt.comm, dbuf + rank, dbuf, 4, st);
            if (!xrc && (cudaMemcpyAsync(all.data(), dbuf, 4 * world, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
                         eng->sync_spin(st) != cudaSuccess))
                xrc = PTAS_ECUDA;
            if (xrc) return xrc;
            acc.s.h2d_bytes += 4;
            acc.s.d2h_bytes += 4 * world;
            for (int q = 0; q < np && q < world; ++q)
                if (all[q] <= XERR) return all[q] - XERR;
            for (int q = 0; q < np; ++q) {
                if (optj[q] < 0) {
                    if (xsrc[q] < 0 || xsrc[q] >= world) return PTAS_EINTERNAL;
                    optj[q] = all[xsrc[q]];
                    if (optj[q] < 0) return PTAS_EINTERNAL;
                    if (opt.memoize && !keys[q].empty()) memo[keys[q]] = optj[q];
                }
                if (xsrc[q] == q && q < world) last_key_of[q] = keys[q];   // rank q holds DP(T_q)
            }
        }
        std::vector<int32_t> f(np);
        for (int q = 0; q < np; ++q) {
            f[q] = optj[q] <= m;
            ptas_probe pr;
            pr.T = Tj[q];
            pr.round = round;
            pr.feasible = f[q];
            pr.K = Kj[q];
            pr.opt = optj[q];
            pr.sigma = sgj[q];
            pr.memo_hit = hit[q];
            pr.rank = who[q];
            plog.push_back(pr);
        }
        interval_update(&LB, &UB, Tj.data(), f.data(), np);
        ++round;
    }

    // ---- a-8 schedule from DP(T*) (readings R9, R11, R12)
    const int64_t Ts = LB;
    hist.classify_full(p, n, Ts, k, &cl);
    std::vector<int64_t> load(m, 0);
    std::vector<int32_t> asg(n, -1);
    int32_t opt_star = 0;
    if (!cl.N.empty()) {
        std::vector<int64_t> key = memo_key(cl, Ts);
        std::vector<MachineCfg> machines;
        DpOutcome tb;
        const double ttb0 = now_s();
        int tslot = -1;
        // MULTI_PROBE: the traceback runs on ONE rank -- the lowest rank whose last DP
        // is DP(T*) (every rank knows which rank computed which probe), else rank 0
        // recomputes it -- and its machine configurations are broadcast
        const bool mp = opt.mode == PTAS_MODE_MULTI_PROBE;
        int owner = 0;
        if (mp)
            for (int r2 = world - 1; r2 >= 0; --r2)
                if (last_key_of[r2] == key) owner = r2;
        if (!mp || rank == owner) {
            for (int b = 0; b < MAX_SLOTS; ++b)
                if (slot_key[b] == key) {
                    tslot = b;
                    break;
                }
            int trc = PTAS_OK;
            if (tslot < 0) {
                DpOutcome ro;
                std::vector<int> order = choose_order(cl.N, cl.r, opt.layout);
                DpRequest rq = make_rq(cl, Ts, opt.mode == PTAS_MODE_LEVEL_SHARDED ? shp : nullptr, order,
                                       (cudaStream_t)opt.stream);
                trc = eng->run_dp(rq, &ro);
                // a recomputation of a DP the search already ran: time, not new work
                acc.s.kernel_launches += ro.launches;
                acc.s.h2d_bytes += ro.h2d;
                acc.s.d2h_bytes += ro.d2h;
                tslot = 0;
            }
            DpSlot *tsl = nullptr;
            if (!trc) trc = eng->slot(tslot, &tsl);
            if (!trc) trc = tsl->traceback(&machines, &tb);
            if (trc && !mp) return trc;
            if (trc) machines.clear(), opt_star = XERR + trc;
            else opt_star = (int32_t)machines.size();
        }
        if (mp) {
            const int Kc = (int)cl.N.size();
            std::vector<int32_t> buf(1 + (size_t)m * Kc, 0);
            buf[0] = opt_star;
            for (size_t mu = 0; mu < machines.size() && (int)mu < m; ++mu)
                std::copy(machines[mu].begin(), machines[mu].end(), buf.begin() + 1 + mu * Kc);
            int32_t *dbuf = nullptr;
            int xrc = eng->exchange_buffer(buf.size() * 4, (void **)&dbuf);
            if (xrc) return xrc;
            cudaStream_t st = opt.stream ? (cudaStream_t)opt.stream : eng->stream();
            if (cudaMemcpyAsync(dbuf, buf.data(), buf.size() * 4, cudaMemcpyHostToDevice, st) != cudaSuccess)
                return PTAS_ECUDA;
            xrc = comm_broadcast(opt.comm, dbuf, buf.size() * 4, owner, st);
            if (xrc) return xrc;
            if (cudaMemcpyAsync(buf.data(), dbuf, buf.size() * 4, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
                eng->sync_spin(st) != cudaSuccess)
                return PTAS_ECUDA;
            if (buf[0] <= XERR) return buf[0] - XERR;
            if (buf[0] < 0 || buf[0] > m) return PTAS_EINTERNAL;
            machines.assign((size_t)buf[0], MachineCfg(Kc));
            for (int32_t mu = 0; mu < buf[0]; ++mu)
                std::copy(buf.begin() + 1 + (size_t)mu * Kc, buf.begin() + 1 + (size_t)(mu + 1) * Kc, machines[mu].begin());
            if (rank != owner) {
                acc.s.h2d_bytes += (int64_t)buf.size() * 4;
                acc.s.d2h_bytes += (int64_t)buf.size() * 4;
            }
        }
        if (std::getenv("PTAS_TRACE"))
            std::fprintf(stderr, "[ptas] traceback at T*=%lld: %zu machines, %.3f ms (slot %d) | host clock %.3f .. %.3f ms\n",
                         (long long)Ts, machines.size(), 1e3 * (now_s() - ttb0), tslot, 1e3 * ttb0, 1e3 * now_s());
        acc.s.kernel_launches += tb.launches;
        acc.s.h2d_bytes += tb.h2d;
        acc.s.d2h_bytes += tb.d2h;
        opt_star = (int32_t)machines.size();
        if ((int)machines.size() > m) return PTAS_EINTERNAL;
        const int K = (int)cl.N.size();
        std::vector<std::vector<int32_t>> jobs_of(K);
        for (int32_t j = 0; j < n; ++j)
            if (cl.cls[j] >= 0) jobs_of[cl.cls[j]].push_back(j);
        std::vector<size_t> next(K, 0);
        for (size_t mu = 0; mu < machines.size(); ++mu)
            for (int i = 0; i < K; ++i)
                for (int32_t t = 0; t < machines[mu][i]; ++t) {
                    if (next[i] >= jobs_of[i].size()) return PTAS_EINTERNAL;
                    int32_t j = jobs_of[i][next[i]++];
                    asg[j] = (int32_t)mu;
                    load[mu] += p[j];
                }
        for (int i = 0; i < K; ++i)
            if (next[i] != jobs_of[i].size()) return PTAS_EINTERNAL;
    }
    // short jobs in input order onto the least loaded machine (lowest index on ties)
    using LI = std::pair<int64_t, int32_t>;
    std::priority_queue<LI, std::vector<LI>, std::greater<LI>> heap;
    for (int32_t q = 0; q < m; ++q) heap.push({load[q], q});
    for (int32_t j = 0; j < n; ++j) {
        if (cl.cls[j] >= 0) continue;
        LI top = heap.top();
        heap.pop();
        asg[j] = top.second;
        load[top.second] += p[j];
        heap.push({load[top.second], top.second});
    }
    int64_t ms = 0;
    for (int32_t q = 0; q < m; ++q) ms = std::max(ms, load[q]);

    *makespan_out = ms;
    std::memcpy(assignment_out, asg.data(), sizeof(int32_t) * n);
    if (log) {
        for (size_t q = 0; q < plog.size() && (int32_t)q < log_cap; ++q) log[q] = plog[q];
    }
    if (log_len) *log_len = (int32_t)plog.size();
    if (stats) {
        acc.s.spec_wasted = (int32_t)spec.size();
        for (auto &kv : spec) acc.interval(kv.second.o);
        acc.finish_wall();
        acc.s.probes = (int32_t)plog.size();
        acc.s.rounds = round;
        acc.s.K_at_Tstar = (int32_t)cl.N.size();
        acc.s.T_star = Ts;
        acc.s.opt_at_Tstar = opt_star;
        acc.s.total_seconds = now_s() - t0;
        *stats = acc.s;
        if (PTAS_KNOB("PTAS_TRACE", 0) == 1)
            std::fprintf(stderr, "[ptas] solve | host clock %.3f .. %.3f ms\n", 1e3 * t0, 1e3 * now_s());
    }
    return PTAS_OK;
}

int validate_dp(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T)
{
    if (K < 0 || K > 64) return PTAS_EINVAL;
    if (K > 0 && (!counts || !sizes)) return PTAS_EINVAL;
    if (T < 1) return PTAS_EINVAL;
    for (int32_t i = 0; i < K; ++i) {
        if (counts[i] < 0 || sizes[i] < 1) return PTAS_EINVAL;
        if (counts[i] > 0 && sizes[i] > T) return PTAS_EINVAL;
    }
    return PTAS_OK;
}

}  // namespace

extern "C" {

void ptas_default_options(ptas_options *o)
{
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->probes_per_round = 1;
    o->mode = PTAS_MODE_SINGLE;
    o->device = -1;
    o->comm = nullptr;
    o->table_budget_bytes = 0;
    o->memoize = 1;
    o->virtual_shards = 1;
    o->layout = 0;
    o->stream = nullptr;
    o->speculate = -1;
    o->shard_min_rows = -1;
    o->window = 0;
}

const char *ptas_strerror(int s)
{
    switch (s) {
    case PTAS_OK: return "ok";
    case PTAS_EINVAL: return "invalid argument";
    case PTAS_ETOOBIG: return "DP table too big (sigma overflow, budget or sum(N) > 65535)";
    case PTAS_ENOMEM: return "out of memory";
    case PTAS_ECUDA: return "CUDA error (no device or kernel failure)";
    case PTAS_ENCCL: return "NCCL unavailable or failed";
    case PTAS_EINTERNAL: return "internal error";
    default: return "unknown status";
    }
}

int ptas_k(double eps) { return k_of(eps); }

int ptas_bounds(const int64_t *p, int32_t n, int32_t m, int64_t *LB, int64_t *UB)
{
    if (!LB || !UB) return PTAS_EINVAL;
    return validate_jobs(p, n, m, LB, UB);
}

int ptas_classify(const int64_t *p, int32_t n, int64_t T, int32_t k, int64_t *u_out, int32_t *K_out,
                  int64_t *r_out, int32_t *N_out, int32_t *cls_out)
{
    if (!p || n < 1 || T < 1 || k < 1 || !u_out || !K_out || !r_out || !N_out || !cls_out)
        return PTAS_EINVAL;
    for (int32_t j = 0; j < n; ++j)
        if (p[j] < 1) return PTAS_EINVAL;
    Classified c;
    classify(p, n, T, k, &c);
    *u_out = c.u;
    *K_out = (int32_t)c.N.size();
    std::memcpy(r_out, c.r.data(), c.r.size() * 8);
    std::memcpy(N_out, c.N.data(), c.N.size() * 4);
    std::memcpy(cls_out, c.cls.data(), (size_t)n * 4);
    return PTAS_OK;
}

int ptas_probe_targets(int64_t LB, int64_t UB, int32_t P, int64_t *out, int32_t *count)
{
    if (!out || !count) return PTAS_EINVAL;
    std::vector<int64_t> v;
    int rc = probe_targets(LB, UB, P, &v);
    if (rc) return rc;
    std::copy(v.begin(), v.end(), out);
    *count = (int32_t)v.size();
    return PTAS_OK;
}

int ptas_interval_update(int64_t *LB, int64_t *UB, const int64_t *T, const int32_t *feasible,
                         int32_t count)
{
    if (!LB || !UB || !T || !feasible || count < 1 || *LB >= *UB) return PTAS_EINVAL;
    interval_update(LB, UB, T, feasible, count);
    return PTAS_OK;
}

int ptas_table_order(const int32_t *counts, const int64_t *sizes, int32_t K, int32_t layout, int32_t *order_out,
                     int32_t *K_out)
{
    if (K < 0 || K > 64 || (K > 0 && (!counts || !sizes || !order_out)) || !K_out || layout < 0 || layout > 1)
        return PTAS_EINVAL;
    for (int32_t i = 0; i < K; ++i)
        if (counts[i] < 0) return PTAS_EINVAL;
    const std::vector<int> o = choose_order(std::vector<int32_t>(counts, counts + K),
                                            std::vector<int64_t>(sizes, sizes + K), layout);
    for (size_t i = 0; i < o.size(); ++i) order_out[i] = o[i];
    *K_out = (int32_t)o.size();
    return PTAS_OK;
}

int ptas_slab_plan(int64_t S, int64_t hi0, int32_t rank, int32_t world, int64_t *pb, int64_t *pe, int64_t *pbase,
                   int64_t *hin, int64_t *hout)
{
    if (world < 1 || rank < 0 || rank >= world || S < world || hi0 < 0 || !pb || !pe || !pbase || !hin || !hout)
        return PTAS_EINVAL;
    slab_plan(S, hi0, rank, world, pb, pe, pbase, hin, hout);
    return PTAS_OK;
}

int ptas_level_shard(int64_t rows, int32_t rank, int32_t world, int64_t row_bytes, int64_t *begin, int64_t *end,
                     int64_t *chunk_out)
{
    if (rows < 0 || world < 1 || rank < 0 || rank >= world || row_bytes < 1 || !begin || !end) return PTAS_EINVAL;
    const int64_t chunk = shard_chunk(rows, world, row_bytes);
    *begin = std::min<int64_t>(rows, (int64_t)rank * chunk);
    *end = std::min<int64_t>(rows, *begin + chunk);
    if (chunk_out) *chunk_out = chunk;
    return PTAS_OK;
}

int ptas_shard_range(int64_t count, int32_t rank, int32_t world, int64_t *begin, int64_t *end)
{
    if (count < 0 || world < 1 || rank < 0 || rank >= world || !begin || !end) return PTAS_EINVAL;
    int64_t chunk = (count + world - 1) / world;
    int64_t b = std::min<int64_t>(count, (int64_t)rank * chunk);
    *begin = b;
    *end = std::min<int64_t>(count, b + chunk);
    return PTAS_OK;
}

int ptas_solve(const int64_t *p, int32_t n, int32_t m, double eps, const ptas_options *opt,
               int64_t *makespan_out, int32_t *assignment_out, ptas_stats *stats)
{
    return solve_core(p, n, m, eps, opt, makespan_out, assignment_out, stats, nullptr, 0, nullptr, 0, 0);
}

int ptas_solve_ex(const int64_t *p, int32_t n, int32_t m, double eps, const ptas_options *opt,
                  int64_t *makespan_out, int32_t *assignment_out, ptas_stats *stats, ptas_probe *log,
                  int32_t log_cap, int32_t *log_len)
{
    return solve_core(p, n, m, eps, opt, makespan_out, assignment_out, stats, log, log_cap, log_len, 0, 0);
}

int ptas_solve_device(const int64_t *d_p, int32_t n, int32_t m, double eps, const ptas_options *opt,
                      int64_t *makespan_out, int32_t *d_assignment, ptas_stats *stats)
{
    if (!d_p || !d_assignment || n < 1) return PTAS_EINVAL;
    int dev;
    int rc = resolve_device(opt ? opt->device : -1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::vector<int64_t> hp(n);
    std::vector<int32_t> ha(n);
    // d_p / d_assignment are read / written on options.stream, or on the legacy
    // default stream when it is NULL (ptas.h): ordered after the work that made p
    // and before the caller's later work on that stream
    {
        std::lock_guard<std::mutex> lk(eng->mu);
        cudaStream_t st = (opt && opt->stream) ? (cudaStream_t)opt->stream : cudaStreamLegacy;
        if (cudaMemcpyAsync(hp.data(), d_p, (size_t)n * 8, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
            eng->sync_spin(st) != cudaSuccess) {
            cudaGetLastError();
            return PTAS_ECUDA;
        }
    }
    rc = solve_core(hp.data(), n, m, eps, opt, makespan_out, ha.data(), stats, nullptr, 0, nullptr,
                    (int64_t)n * 4, (int64_t)n * 8);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    cudaStream_t st = (opt && opt->stream) ? (cudaStream_t)opt->stream : cudaStreamLegacy;
    if (cudaMemcpyAsync(d_assignment, ha.data(), (size_t)n * 4, cudaMemcpyHostToDevice, st) != cudaSuccess ||
        eng->sync_spin(st) != cudaSuccess) {
        cudaGetLastError();
        return PTAS_ECUDA;
    }
    return PTAS_OK;
}

int dp_table_shape(const int32_t *counts, int32_t K, int64_t *sigma_out, int32_t *elem_bytes_out)
{
    if (K < 0 || K > 64 || (K > 0 && !counts) || !sigma_out || !elem_bytes_out) return PTAS_EINVAL;
    __int128 sg = 1;
    int64_t sumN = 0;
    for (int32_t i = 0; i < K; ++i) {
        if (counts[i] < 0) return PTAS_EINVAL;
        sumN += counts[i];
    }
    for (int32_t i = 0; i < K; ++i) {
        sg *= (__int128)counts[i] + 1;
        if (sg > (__int128)INT64_MAX) return PTAS_ETOOBIG;
    }
    if (sumN > 65535) return PTAS_ETOOBIG;
    *sigma_out = (int64_t)sg;
    *elem_bytes_out = sumN <= 255 ? 1 : 2;
    return PTAS_OK;
}

static int dp_fill_common(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T,
                          void *d_ext, int64_t ext_bytes, cudaStream_t st, void *host_out,
                          int64_t host_bytes, int32_t *opt_N_out, ptas_stats *stats)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    const double t0 = now_s();
    int rc = validate_dp(counts, sizes, K, T);
    if (rc) return rc;
    if (!opt_N_out) return PTAS_EINVAL;
    int64_t sigma;
    int32_t e;
    rc = dp_table_shape(counts, K, &sigma, &e);
    if (rc) return rc;
    if (host_out && host_bytes < sigma * e) return PTAS_EINVAL;
    if (d_ext && ext_bytes < sigma * e) return PTAS_EINVAL;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    DpRequest rq;
    rq.K = K;
    rq.N = counts;
    rq.r = sizes;
    rq.T = T;
    rq.ext_table = d_ext;
    rq.ext_bytes = ext_bytes;
    rq.stream = st;
    DpOutcome o;
    rc = eng->run_dp(rq, &o);
    if (rc) return rc;
    Acc acc;
    acc.add(o);
    acc.s.fill_wall_seconds = o.fill_s;
    if (host_out) {
        // engine-owned table; identity order => caller's layout
        rc = eng->copy_table_to_host(host_out, sigma * e);
        if (rc) return rc;
        acc.s.d2h_bytes += sigma * e;
    }
    *opt_N_out = o.opt;
    if (stats) {
        acc.s.unique_dps = 1;
        acc.s.total_seconds = now_s() - t0;
        *stats = acc.s;
    }
    return PTAS_OK;
}

int dp_fill_opt(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, int64_t table_budget_bytes,
                int32_t window, int32_t *opt_N_out, ptas_stats *stats)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    const double t0 = now_s();
    int rc = validate_dp(counts, sizes, K, T);
    if (rc) return rc;
    if (!opt_N_out || window < -1 || window > 1 || table_budget_bytes < 0) return PTAS_EINVAL;
    int64_t sigma;
    int32_t e;
    rc = dp_table_shape(counts, K, &sigma, &e);
    if (rc) return rc;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    const std::vector<int32_t> N(counts, counts + K);
    const std::vector<int64_t> r(sizes, sizes + K);
    const std::vector<int> full = choose_order(N, r, 0), win = window_order(N, r, T);
    DpRequest rq;
    rq.K = K;
    rq.N = counts;
    rq.r = sizes;
    rq.T = T;
    rq.budget = table_budget_bytes;
    DpOutcome o;
    rc = PTAS_ETOOBIG;
    if (window <= 0) {
        rq.order = full.data();
        rc = eng->run_dp(rq, &o);
    }
    if (rc == PTAS_ETOOBIG && window >= 0) {
        rq.order = win.data();
        rq.window = 1;
        rc = eng->run_dp(rq, &o);
        if (rc == PTAS_ETOOBIG && window == 1) {   // the window saves nothing: full table
            rq.order = full.data();
            rq.window = 0;
            rc = eng->run_dp(rq, &o);
        }
    }
    if (rc) return rc;
    Acc acc;
    acc.add(o);
    acc.s.fill_wall_seconds = o.fill_s;
    *opt_N_out = o.opt;
    if (stats) {
        acc.s.unique_dps = 1;
        acc.s.total_seconds = now_s() - t0;
        *stats = acc.s;
    }
    return PTAS_OK;
}

int dp_fill_alg4(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, int32_t dim, void *table_out,
                 int64_t table_bytes, int32_t *opt_N_out, int32_t *divisor_out, ptas_stats *stats)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    const double t0 = now_s();
    int rc = validate_dp(counts, sizes, K, T);
    if (rc) return rc;
    if (!opt_N_out || K < 1 || K > 16 || dim < 1) return PTAS_EINVAL;
    int64_t sigma;
    int32_t e;
    rc = dp_table_shape(counts, K, &sigma, &e);
    if (rc) return rc;
    if (table_out && table_bytes < sigma * e) return PTAS_EINVAL;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    DpRequest rq;
    rq.K = K;
    rq.N = counts;
    rq.r = sizes;
    rq.T = T;
    std::vector<int32_t> dig;
    int64_t nC = 0;
    rc = eng->configs_canonical(rq, &dig, &nC);   // C(T), caller order (enumerated on the device)
    if (rc) return rc;
    ptas_stats st;
    std::memset(&st, 0, sizeof(st));
    for (int64_t c = 0; c < nC; ++c) {   // closed-form relaxation count
        double pr = 1;
        for (int i = 0; i < K; ++i) pr *= (double)(counts[i] - dig[(size_t)c * K + i] + 1);
        st.relaxations += pr;
    }
    double fs = 0;
    int64_t nb = 0;
    int32_t bl = 0;
    int32_t divs[16];
    if (nC == 0) {   // no long class: OPT(0) = 0 only
        *opt_N_out = 0;
    } else {
        rc = alg4_fill(e, counts, K, dig.data(), nC, dim, table_out, opt_N_out, &fs, &nb, &bl, divs);
        if (rc) return rc;
    }
    if (divisor_out) std::memcpy(divisor_out, divs, sizeof(int32_t) * K);
    if (stats) {
        st.unique_dps = 1;
        st.fill_seconds = st.fill_wall_seconds = fs;
        st.states = sigma;
        st.sigma_max = sigma;
        st.relax_executed = st.relaxations;
        st.alg_bytes = st.exec_bytes = (st.relaxations + (double)sigma) * e;
        st.fill_launches = bl;
        st.total_seconds = now_s() - t0;
        st.opt_at_Tstar = *opt_N_out;
        *stats = st;
    }
    return PTAS_OK;
}

int hmbp_solve(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t capacity, int32_t *bins_out,
               int32_t *packing_out, int32_t max_bins, ptas_stats *stats)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    const double t0 = now_s();
    int rc = validate_dp(counts, sizes, K, capacity);
    if (rc) return rc;
    if (!bins_out) return PTAS_EINVAL;
    int64_t total = 0;
    std::vector<int32_t> N(counts, counts + K);
    for (int32_t x : N) total += x;
    if (packing_out && max_bins < total) return PTAS_EINVAL;
    Acc acc;
    if (total == 0) {
        *bins_out = 0;
        if (stats) {
            acc.s.total_seconds = now_s() - t0;
            *stats = acc.s;
        }
        return PTAS_OK;
    }
    int64_t sigma;
    int32_t e;
    rc = dp_table_shape(counts, K, &sigma, &e);
    if (rc) return rc;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    // internal layout of the solve (D2, D13)
    std::vector<int> order = choose_order(N, std::vector<int64_t>(sizes, sizes + K), 0);
    DpRequest rq;
    rq.K = K;
    rq.N = counts;
    rq.r = sizes;
    rq.T = capacity;
    rq.order = order.data();
    DpOutcome o;
    rc = eng->run_dp(rq, &o);
    if (rc) return rc;
    acc.add(o);
    acc.s.fill_wall_seconds = o.fill_s;
    std::vector<MachineCfg> bins;   // canonical (caller-order) digit vectors, traceback order
    DpOutcome tb;
    rc = eng->traceback(&bins, &tb);
    if (rc) return rc;
    if ((int32_t)bins.size() != o.opt) return PTAS_EINTERNAL;
    acc.s.kernel_launches += tb.launches;
    acc.s.h2d_bytes += tb.h2d;
    acc.s.d2h_bytes += tb.d2h;
    if (packing_out)
        for (size_t b = 0; b < bins.size(); ++b)
            for (int i = 0; i < K; ++i) packing_out[(int64_t)b * K + i] = bins[b][i];
    *bins_out = o.opt;
    if (stats) {
        acc.s.unique_dps = 1;
        acc.s.opt_at_Tstar = o.opt;
        acc.s.total_seconds = now_s() - t0;
        *stats = acc.s;
    }
    return PTAS_OK;
}

int dp_fill(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, void *table_out,
            int64_t table_bytes, int32_t *opt_N_out, ptas_stats *stats)
{
    return dp_fill_common(counts, sizes, K, T, nullptr, 0, nullptr, table_out, table_bytes, opt_N_out,
                          stats);
}

int dp_fill_device(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, void *d_table,
                   int64_t table_bytes, void *cuda_stream, int32_t *opt_N_out)
{
    if (!d_table) return PTAS_EINVAL;
    // NULL = the legacy default stream (ptas.h): ordered after the caller's work on it
    return dp_fill_common(counts, sizes, K, T, d_table, table_bytes,
                          cuda_stream ? (cudaStream_t)cuda_stream : cudaStreamLegacy, nullptr, 0, opt_N_out,
                          nullptr);
}

int dp_configs(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, int32_t *out_digits,
               int64_t cap, int64_t *count)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    int rc = validate_dp(counts, sizes, K, T);
    if (rc) return rc;
    if (!count || (cap > 0 && !out_digits)) return PTAS_EINVAL;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    DpRequest rq;
    rq.K = K;
    rq.N = counts;
    rq.r = sizes;
    rq.T = T;
    std::vector<int32_t> dig;
    int64_t c = 0;
    rc = eng->configs_canonical(rq, &dig, &c);
    if (rc) return rc;
    *count = c;
    if (out_digits && cap >= c) std::copy(dig.begin(), dig.end(), out_digits);
    return PTAS_OK;
}

int dp_row_index(const int32_t *counts, int32_t K, int64_t *level_start, int64_t level_cap,
                 int64_t *out_rowbase, int64_t rows_cap)
{
    knobs_refresh();   // PTAS_* knobs: re-read at most once per call
    if (K < 1 || K > 64 || !counts || !level_start) return PTAS_EINVAL;
    int64_t sigma;
    int32_t e;
    int rc = dp_table_shape(counts, K, &sigma, &e);
    if (rc) return rc;
    int dev;
    rc = resolve_device(-1, &dev);
    if (rc) return rc;
    Engine *eng;
    rc = Engine::get(dev, &eng);
    if (rc) return rc;
    std::lock_guard<std::mutex> lk(eng->mu);
    std::vector<int64_t> ls, rb;
    rc = eng->row_index(counts, K, &ls, &rb);
    if (rc) return rc;
    if ((int64_t)ls.size() > level_cap) return PTAS_EINVAL;
    std::copy(ls.begin(), ls.end(), level_start);
    if (out_rowbase) {
        if ((int64_t)rb.size() > rows_cap) return PTAS_EINVAL;
        std::copy(rb.begin(), rb.end(), out_rowbase);
    }
    return PTAS_OK;
}

}  // extern "C"
