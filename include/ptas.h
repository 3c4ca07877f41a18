/*
 * ptas.h — C ABI of the B200-native PTAS hot path (libptas_b200.so).
 *
 * Method: Li, Ghalami, Schwiebert, Grosu, "A GPU Parallel Approximation
 * Algorithm for Scheduling Parallel Identical Machines to Minimize
 * Makespan", IPDPS workshops 2018.  Citations are
 * PAPER.md:<line> (section / algorithm / equation).
 *
 * Conventions (all entry points):
 *  - Every function returns an int status: PTAS_OK (0) or a negative
 *    PTAS_E* code; ptas_strerror() names it.  On error nothing partial is
 *    written to any output argument.
 *  - Ownership: the caller owns every pointer argument.  The library never
 *    frees caller memory and keeps no pointer after a call returns (except
 *    the opaque ptas_comm it creates, released by ptas_comm_destroy).
 *    Device workspace is allocated and cached internally per device.
 *  - Host pointers are ordinary (pageable or pinned) host memory; "device"
 *    pointers are CUDA global-memory pointers on the current device
 *    (e.g. torch.Tensor.data_ptr()).
 *  - Table layout: row-major over the classes in the order given, last
 *    class fastest, elem_bytes per entry (1 = uint8 when sum(counts) <= 255,
 *    else 2 = uint16; OPT(n) <= sum(n) so the value always fits).
 *  - Determinism: outputs are a pure function of the inputs and
 *    probes_per_round; they do not depend on mode or GPU count.
 *  - Thread safety: calls on different devices may run concurrently; calls
 *    on one device are serialised by an internal per-device lock.
 */
#ifndef PTAS_B200_H
#define PTAS_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
    PTAS_OK = 0,
    PTAS_EINVAL = -1,     /* invalid argument (see each function)              */
    PTAS_ETOOBIG = -2,    /* sigma overflows / exceeds the table budget,
                             sum(counts) > 65535, or digits do not pack        */
    PTAS_ENOMEM = -3,     /* device or host allocation failed                  */
    PTAS_ECUDA = -4,      /* CUDA runtime error (no device, launch failure)    */
    PTAS_ENCCL = -5,      /* NCCL missing or failed                            */
    PTAS_EINTERNAL = -6   /* internal invariant violated (a bug)               */
};

enum {
    PTAS_MODE_SINGLE = 0,        /* one GPU                                          */
    PTAS_MODE_LEVEL_SHARDED = 1, /* each row-level split over the ranks of comm,
                                    slices NCCL all-gathered         */
    PTAS_MODE_MULTI_PROBE = 2    /* one T probe per rank per round (Alg 3 quarter
                                    split generalised)            */
};

typedef struct ptas_comm ptas_comm; /* opaque; wraps an ncclComm_t */

typedef struct {
    int32_t probes_per_round;   /* P >= 1; 1 = Alg 1 bisection (default).  In
                                   MULTI_PROBE mode it must equal the comm size. */
    int32_t mode;               /* PTAS_MODE_*                                     */
    int32_t device;             /* CUDA device (-1 = current)                      */
    ptas_comm *comm;            /* NULL = single GPU                               */
    int64_t table_budget_bytes; /* 0 = auto: free HBM minus a 2 GiB reserve        */
    int32_t memoize;            /* 1 (default) reuse OPT(N) across equal DP keys   */
    int32_t virtual_shards;     /* >1 with mode LEVEL_SHARDED and comm == NULL:
                                   run that many logical shards on one GPU
                                   (slice + gather + scatter), for testing          */
    int32_t layout;             /* 0 = internal class order chosen by the library
                                   (largest count fastest); 1 = classes in
                                   ascending-size order as classified             */
    void *stream;               /* cudaStream_t for all device work of the call
                                   (NULL = the library's own stream); the call
                                   still returns only when its work is done       */
    int32_t speculate;          /* P = 1, SINGLE mode: evaluate upcoming probes of
                                   Alg 1 concurrently while the DPs are small
                                   (-1 = library default: the next 4 probes on
                                   the all-feasible path; 0 = off; d > 0 = the
                                   whole bisection tree d levels deep, up to
                                   2^d - 1 probes in flight).  The probe
                                   sequence, T* and the schedule are those of
                                   Alg 1 (D8); only time changes.      */
    int32_t window;             /* level window for feasibility probes (DESIGN.md
                                   D15): 0 = when a probe's full
                                   table exceeds the budget (default), 1 = for
                                   every probe DP, -1 = never.  Only OPT(N) of a
                                   windowed DP is kept; the schedule's DP at T* is
                                   always a full table (ETOOBIG if it does not fit) */
    int32_t slab_pipeline;      /* LEVEL_SHARDED with comm, windowed probe DPs
                                   (window = 1, or a table over the budget):
                                   0 = the window's slabs split over the ranks and
                                   all-gathered (default); 1 = the slab/halo
                                   pipeline of SURVEY.md §8(f)-2ii: rank g holds a
                                   contiguous range of slabs of the first internal
                                   class (the table split along that dimension,
                                   plus min(N0, T/r0) halo slabs), fills them in
                                   chunks of the other classes' levels, and sends
                                   the halo of each chunk to rank g + 1 with
                                   ncclSend / ncclRecv (a wavefront over ranks and
                                   chunks); OPT(N) is broadcast from the last rank */
    int64_t shard_min_rows;     /* LEVEL_SHARDED with comm: row-levels with fewer
                                   rows are computed redundantly on every rank
                                   (-1 = library default 2048); 0 = shard every
                                   row-level, also at world size 1 (the slice /
                                   ncclAllGather / scatter path on one GPU)      */
} ptas_options;

typedef struct {
    int32_t probes, rounds, unique_dps, K_at_Tstar;
    int64_t T_star, sigma_max, opt_at_Tstar;
    double relaxations;     /* closed-form (n,s) pairs over executed DPs       */
    double dp_seconds;      /* device time of all DP work (CUDA events)        */
    double fill_seconds;    /* device time of the level-fill loops             */
    double total_seconds;   /* host wall time of the call                      */
    double alg_bytes;       /* level-fill algorithmic bytes: sum (relax+sigma)*e */
    int64_t states;         /* sum of sigma over executed DPs                  */
    int32_t kernel_launches;/* kernels launched by the library in this call    */
    int32_t fill_launches;  /* of which level-fill launches                    */
    int64_t h2d_bytes, d2h_bytes; /* host<->device bytes moved by this call    */
    double relax_executed;  /* (n, s') relaxations the fill kernels evaluated:
                               the packed kernel takes one window per prefix
                               s' (reading D5), so this is below
                               `relaxations`; equal on the scalar kernel      */
    double exec_bytes;      /* sum (relax_executed + sigma) * e: the table bytes
                               the fill kernels gather and write              */
    int32_t spec_dps;       /* DPs evaluated speculatively (options.speculate) */
    int32_t spec_wasted;    /* of which never probed by the search (their work
                               is not counted in the fields above)            */
    double fill_wall_seconds; /* device time during which at least one level-
                               fill loop ran: union of the DPs' fill intervals
                               (CUDA events on one time axis).  Equals
                               fill_seconds when DPs run one at a time; below it
                               when speculative / concurrent DPs overlap       */
    int32_t window_dps;     /* DPs run in level-window mode (D15)     */
    int32_t pad_;
    int64_t dev_bytes_max;  /* largest device memory of one DP: table (or the
                               window's resident slabs) + row index            */
} ptas_stats;

typedef struct {
    int64_t T;        /* probe target makespan                              */
    int32_t round;    /* search round (0-based)                             */
    int32_t feasible; /* OPT(N) <= m                                        */
    int32_t K;        /* non-empty classes at T                             */
    int32_t opt;      /* OPT(N) (0 if no long job)                          */
    int64_t sigma;    /* DP table size prod(N_i+1)                          */
    int32_t memo_hit; /* 1 if OPT(N) came from the memo                     */
    int32_t rank;     /* rank that evaluated the probe (MULTI_PROBE)        */
} ptas_probe;

/* Default options (P = 1, SINGLE, current device, memoize, auto budget). */
void ptas_default_options(ptas_options *opt);

/* ---------------------------------------------------------------- solve
 * PTAS for P||Cmax — Alg 1 with the P-probe search of
 * Alg 3 (reading R8 in DESIGN.md), the k-dimensional DP
 * of Eq. 1 on the GPU per probe, and the schedule from
 * DP(T*) with short jobs placed greedily.
 *   p[n]       host, processing times, each >= 1
 *   n >= 1, m >= 1, eps > 0 finite (k = ceil(1/eps))
 *   opt        nullable (defaults)
 *   makespan_out  host int64, the schedule's makespan (actual sizes)
 *   assignment_out host int32[n], machine 0..m-1 of each job
 *   stats      nullable
 * EINVAL: n<1, m<1, eps<=0 or non-finite, any p<1, sum(p) overflow,
 *         P<1, bad mode/comm combination.  ETOOBIG: a probe's DP table
 *         exceeds the budget. */
int ptas_solve(const int64_t *p, int32_t n, int32_t m, double eps,
               const ptas_options *opt, int64_t *makespan_out,
               int32_t *assignment_out, ptas_stats *stats);

/* As ptas_solve, plus the probe log (log nullable, log_cap entries;
 * *log_len = number of probes, which may exceed log_cap). */
int ptas_solve_ex(const int64_t *p, int32_t n, int32_t m, double eps,
                  const ptas_options *opt, int64_t *makespan_out,
                  int32_t *assignment_out, ptas_stats *stats,
                  ptas_probe *log, int32_t log_cap, int32_t *log_len);

/* Device-resident variant: d_p (int64[n]) and d_assignment (int32[n]) are
 * device pointers on the chosen device; makespan_out is host.  The host
 * driver stages p to host memory internally (counted in stats->d2h_bytes).
 * d_p is read and d_assignment written on options->stream, or on the legacy
 * default stream when it is NULL, so both are ordered with the caller's work
 * on that stream; the call returns when d_assignment is written. */
int ptas_solve_device(const int64_t *d_p, int32_t n, int32_t m, double eps,
                      const ptas_options *opt, int64_t *makespan_out,
                      int32_t *d_assignment, ptas_stats *stats);

/* ---------------------------------------------------------------- DP
 * sigma = prod(counts[i]+1) (Alg 2 l.2) and the entry size.
 * EINVAL: K<0, K>64, counts[i]<0.  ETOOBIG: sigma overflows int64 or
 * sum(counts) > 65535. */
int dp_table_shape(const int32_t *counts, int32_t K, int64_t *sigma_out,
                   int32_t *elem_bytes_out);

/* Fill the whole DP table of Eq. 1:
 *   OPT(0) = 0,  OPT(n) = 1 + min_{s in C(T), s <= n} OPT(n - s),
 *   C(T) = { s != 0 : 0 <= s_i <= counts_i, sum s_i sizes_i <= T }
 * (Alg 2 l.17).  counts/sizes are host arrays of length K in
 * the class order the table is laid out in.
 *   table_out  host, nullable ("just OPT(N)"), table_bytes >= sigma*e
 *   opt_N_out  host int32, OPT(counts)
 *   stats      nullable (relaxations, fill_seconds, ...)
 * EINVAL: K<0 or >64, counts<0, sizes<1, T<1, a size > T with count > 0,
 *         table_out != NULL with table_bytes < sigma*e.  ETOOBIG as
 *         dp_table_shape or sigma*e over the budget.  K = 0 gives
 *         sigma = 1 and OPT = 0. */
int dp_fill(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T,
            void *table_out, int64_t table_bytes, int32_t *opt_N_out,
            ptas_stats *stats);

/* OPT(N) of Eq. 1 only (no table), with the level window of SURVEY.md
 * §8(f)-2i / DESIGN.md D15 when the full table does not fit: rows whose first
 * internal class count p0 is >= 1 depend only on the slabs p0 - s0 (1 <= s0 <=
 * min(N0, T / r0)), so only those slabs are resident (a ring mapped twice in
 * virtual memory) and the table can exceed the device memory by the factor
 * (N0 + 1) / (min(N0, T / r0) + 1) ("only the values of the
 * subproblems in these blocks are needed on the GPU").
 *   counts, sizes, K, T : as dp_fill (caller order; the library picks the
 *                         internal order, the result does not depend on it)
 *   table_budget_bytes  : device bytes the DP may use (0 = free HBM - 2 GiB)
 *   window              : 0 = only when the full table exceeds the budget,
 *                         1 = always (when it saves memory), -1 = never
 *   opt_N_out           : host int32, OPT(counts)
 *   stats               : nullable (window_dps = 1 when windowed,
 *                         dev_bytes_max = device bytes used)
 * EINVAL as dp_fill; ETOOBIG when even the window exceeds the budget, or the
 * window saves nothing (min(N0, T / r0) >= N0 for every class) and the full
 * table does not fit. */
int dp_fill_opt(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T,
                int64_t table_budget_bytes, int32_t window, int32_t *opt_N_out,
                ptas_stats *stats);

/* The paper's own DP design as an A/B baseline: the
 * data-partitioning scheme of Alg 4 / Alg 5 --
 * divisor per dimension (floor(sqrt(n_i + 1)) lowered until it divides n_i + 1,
 * only the `dim` largest kept), the table reorganised into blocks stored
 * consecutively, block-levels in order with the blocks of a level
 * concurrently (one CTA each), in-block anti-diagonal levels in order, every
 * entry relaxed over every configuration s <= v.  Same values as dp_fill.
 *   counts, sizes, K (1..16), T : as dp_fill;  dim >= 1 (the paper used 3..9)
 *   table_out   : host, nullable; row-major in the caller's order (converted
 *                 back from the blocked layout), table_bytes >= sigma * e
 *   opt_N_out   : host int32, OPT(counts)
 *   divisor_out : host int32[K], nullable: the divisor used
 *   stats       : nullable (fill_seconds = device time of the block-levels,
 *                 fill_launches = block-levels, relaxations = Eq. 1 count)
 * Errors as dp_fill; ETOOBIG when a block exceeds 2^31 entries or the
 * per-CTA tables exceed shared memory. */
int dp_fill_alg4(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t T, int32_t dim,
                 void *table_out, int64_t table_bytes, int32_t *opt_N_out, int32_t *divisor_out,
                 ptas_stats *stats);

/* High-multiplicity bin packing on the same level-fill engine (SURVEY.md
 * §8(f)-4; the paper's future work on other higher-dimensional DPs,
 * PAPER.md:472).  Eq. 1 with T = capacity and r = sizes is
 * exactly this problem: OPT(N) is the minimum number of bins of capacity
 * `capacity` that hold counts[i] items of size sizes[i].
 *   counts[K], sizes[K] : host arrays (caller order; zero counts allowed)
 *   bins_out            : host, receives OPT(N) (minimum number of bins)
 *   packing_out         : host, nullable; [max_bins][K] int32, row b = items
 *                         of each class in bin b, bins in traceback order
 *                         (reading R11: first configuration in lexicographic
 *                         order of the caller's class order)
 *   max_bins            : rows of packing_out; must be >= sum(counts)
 *   stats               : nullable, as dp_fill (+ traceback launches)
 * The table is laid out internally by ascending count (D2); the
 * result does not depend on it.  Errors: as dp_fill (EINVAL for a size >
 * capacity with a positive count, capacity < 1, ...), EINVAL if packing_out
 * is given with max_bins < sum(counts).  Nothing is written on error. */
int hmbp_solve(const int32_t *counts, const int64_t *sizes, int32_t K, int64_t capacity,
               int32_t *bins_out, int32_t *packing_out, int32_t max_bins, ptas_stats *stats);

/* As dp_fill, into a caller-owned device buffer d_table (>= sigma*e bytes,
 * e.g. a torch uint8/uint16 tensor) on the current device, enqueued on
 * cuda_stream (a cudaStream_t; NULL = legacy default stream).  The call
 * synchronises the stream once at the end to read OPT(N). */
int dp_fill_device(const int32_t *counts, const int64_t *sizes, int32_t K,
                   int64_t T, void *d_table, int64_t table_bytes,
                   void *cuda_stream, int32_t *opt_N_out);

/* ---------------------------------------------------------------- multi-GPU
 * NCCL communicator over NVLink for LEVEL_SHARDED / MULTI_PROBE modes.  One
 * process per GPU; the 128-byte unique id is made on rank 0 and broadcast
 * by the caller (e.g. torch.distributed).  NCCL is loaded at run time
 * (libnccl.so.2); PTAS_ENCCL if it is absent. */
int ptas_get_unique_id(void *out128);
int ptas_comm_init(ptas_comm **c, int32_t rank, int32_t world,
                   const void *unique_id128, int32_t device);
int ptas_comm_destroy(ptas_comm *c);

const char *ptas_strerror(int status);

/* ---------------------------------------------------------------- host steps
 * The host-side steps of the driver, exported so they can be checked on a
 * machine without a GPU.  Pure functions, no CUDA calls. */

/* k = ceil(1/eps).  Returns k, or PTAS_EINVAL. */
int ptas_k(double eps);
/* LB, UB of Alg 1 l.2-3. */
int ptas_bounds(const int64_t *p, int32_t n, int32_t m, int64_t *LB, int64_t *UB);
/* Long/short split and rounding of Alg 1 l.6-8:
 * u = max(1, floor(T/k^2)), long iff k*p > T, r = floor(p/u)*u, classes =
 * distinct r ascending.  r_out, N_out have room for n; cls_out[n] = class
 * or -1 (short). */
int ptas_classify(const int64_t *p, int32_t n, int64_t T, int32_t k,
                  int64_t *u_out, int32_t *K_out, int64_t *r_out,
                  int32_t *N_out, int32_t *cls_out);
/* Probe targets of one round: T_j = LB + floor((2j+1)(UB-LB)/(2P)),
 * deduplicated (out has room for P).  EINVAL if LB >= UB or P < 1. */
int ptas_probe_targets(int64_t LB, int64_t UB, int32_t P, int64_t *out,
                       int32_t *count);
/* Interval update after a round (Alg 1 l.10-14 for P = 1; Alg 3 l.13-25
 * as read in DESIGN.md R8). */
int ptas_interval_update(int64_t *LB, int64_t *UB, const int64_t *T,
                         const int32_t *feasible, int32_t count);
/* Contiguous slice [begin, end) of `count` items owned by `rank` of
 * `world` (ceil split; trailing ranks may be empty). */
int ptas_shard_range(int64_t count, int32_t rank, int32_t world,
                     int64_t *begin, int64_t *end);
/* Slab/halo pipeline plan (ptas_options.slab_pipeline):
 * S = N0 + 1 slabs of the first internal class over `world` ranks; rank
 * `rank` owns slabs [*pb, *pe), holds [*pbase, *pe) (its *hin halo slabs are
 * received per chunk from rank - 1), and sends the chunk rows of its last
 * *hout slabs to rank + 1 (hin of rank g == hout of rank g - 1).  hi0 =
 * min(N0, T / r0).  Host only; the engine uses exactly this plan.
 * EINVAL: S < world, world < 1, rank outside [0, world), hi0 < 0. */
int ptas_slab_plan(int64_t S, int64_t hi0, int32_t rank, int32_t world, int64_t *pb, int64_t *pe,
                   int64_t *pbase, int64_t *hin, int64_t *hout);

/* The split the level-sharded DP uses for one row-level of `rows` rows of
 * `row_bytes` bytes each (rows of a level are independent,
 * PAPER.md:215): ceil(rows / world) rounded up to the smallest multiple q with
 * q * row_bytes = 0 (mod 16), so every rank's compact slice starts 16-byte
 * aligned; rank r owns [min(rows, r*chunk), min(rows, (r+1)*chunk)), trailing
 * ranks may be empty.  *chunk_out (nullable) = the per-rank slice length every
 * rank contributes to the ncclAllGather (padded).  EINVAL: rows < 0,
 * world < 1, rank outside [0, world), row_bytes < 1, null begin/end. */
int ptas_level_shard(int64_t rows, int32_t rank, int32_t world, int64_t row_bytes,
                     int64_t *begin, int64_t *end, int64_t *chunk_out);

/* Internal class order of the DP table (D2,
 * D13): order_out[i] = the caller class laid out at position i (the
 * non-empty classes only, *K_out of them; position K_out - 1 is the
 * contiguous row dimension).  layout 0 (ptas_solve's default, options.layout):
 * the largest-count class last, the others by descending size; layout 1: the
 * given order.  ptas_solve lays out every probe's table this way, so
 * dp_fill(counts[order], sizes[order]) computes the solve's own layout.
 *   counts[K], sizes[K] host; order_out host int32[K] (room for K).
 * EINVAL: K < 0 or > 64, counts < 0, null pointers, layout not 0/1.
 * Pure host function (no CUDA). */
int ptas_table_order(const int32_t *counts, const int64_t *sizes, int32_t K,
                     int32_t layout, int32_t *order_out, int32_t *K_out);

/* ---------------------------------------------------------------- inspection
 * Device steps exposed for parity tests (need a GPU). */

/* Configuration set C(T) as enumerated by the device kernel, canonical
 * lexicographic order; out_digits[count*K] (nullable when cap == 0). */
int dp_configs(const int32_t *counts, const int64_t *sizes, int32_t K,
               int64_t T, int32_t *out_digits, int64_t cap, int64_t *count);
/* Row-level index (level structure over the K-1 leading classes):
 * level_start[rho_max+2] prefix sums of row counts per row-level and, for
 * every row slot in row-level order, its table offset (row base index).
 * out_rowbase has room for sigma / (counts[K-1]+1) entries (nullable). */
int dp_row_index(const int32_t *counts, int32_t K, int64_t *level_start,
                 int64_t level_cap, int64_t *out_rowbase, int64_t rows_cap);

#ifdef __cplusplus
}
#endif
#endif /* PTAS_B200_H */
