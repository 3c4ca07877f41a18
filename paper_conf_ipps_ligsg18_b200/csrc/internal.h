// internal.h — shared declarations of the product library (NOT used by oracle/).
//
// Layout of a DP in HBM:
//   table  : entries of E (uint8 if sum N <= 255 else uint16), row-major over
//            the INTERNAL class order (a permutation of the caller's order
//            chosen by the driver; identity for dp_fill), last class fastest.
//            A "row" is the run of W = N[K-1]+1 entries that share the K1 = K-1
//            leading digits p; rows are stored with pitch Wp (W*e rounded up
//            to a multiple of 4 bytes, and of 4*CH bytes for rows of 8 or
//            more words, CH = the fill kernel's words per lane) so every row
//            and every off(s') is aligned for the kernel's vector loads.  Rows are filled in row-level order rho = sum(p) (the
//            wavefront).  The caller's layout (pitch W) is produced by a
//            compaction copy when Wp != W.
//   configs: C(T) in internal lexicographic order: uint16
//            digits [nC*K] + int64 linear offsets off(s) [nC].
//   prefix : one entry per distinct leading part s' of C (runs of equal s' in
//            lexicographic order): packed digits, off(s'), Jmax(s') = largest
//            last digit with (s', j) in C.  Entry 0 is s' = 0 (j = 1..J0).
#pragma once
#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

namespace ptas {

// Tuning / test knobs (PTAS_* environment variables; the defaults are the
// measured best).  Every C-ABI entry point calls knobs_refresh(), and
// each PTAS_KNOB call site re-reads its variable only when the generation has
// changed: no getenv per launch or per level, while tests can still change a
// knob between calls.  Unset or empty -> DFLT.
uint64_t knob_generation();
void knobs_refresh();
#define PTAS_KNOB(NAME, DFLT)                                                                    \
    ([]() -> int64_t {                                                                             \
        static std::atomic<uint64_t> g_{~0ull};                                                    \
        static std::atomic<int64_t> v_{0};                                                          \
        const uint64_t cur_ = ::ptas::knob_generation();                                           \
        if (g_.load(std::memory_order_acquire) != cur_) {                                          \
            const char *t_ = std::getenv(NAME);                                                    \
            v_.store(t_ && t_[0] ? (int64_t)std::atoll(t_) : (int64_t)(DFLT), std::memory_order_relaxed); \
            g_.store(cur_, std::memory_order_release);                                             \
        }                                                                                          \
        return v_.load(std::memory_order_relaxed);                                                 \
    }())

constexpr int MAXK = 40;   // internal (non-empty) classes
constexpr int MAXW = 2;    // 64-bit words for packed leading digits

struct PrefixEntry {
    uint64_t w[MAXW];   // packed leading digits s'
    int64_t off;        // sum_i s'_i * stride_i (elements)
    int32_t jmax;       // max j with (s', j) in C
    int32_t pad;
};
static_assert(sizeof(PrefixEntry) == 32, "PrefixEntry must be 32 bytes");

// Geometry of the row space, passed by value to the kernels.
struct RowGeom {
    int32_t K1;                 // number of leading classes (K-1)
    int32_t rho_max;            // sum of leading counts
    int64_t W;                  // row length N[K-1]+1
    int64_t Wp;                 // padded row pitch (entries), see row_pitch_words()
    int32_t N[MAXK];            // leading counts
    int32_t maxsuf[MAXK + 1];   // maxsuf[i] = sum_{d >= i} N[d] (leading dims)
    int64_t stride[MAXK];       // element strides of the leading dims
    uint8_t word[MAXK];         // packed word index of leading digit i
    uint8_t shift[MAXK];        // bit offset of leading digit i
    uint64_t guard[MAXW];       // guard bit per field, per word
    uint64_t maxs[MAXW];        // packed hi_i = min(N_i, T / r_i): the digit-wise max over the prefixes of C(T)
    int32_t nwords;
    // dominance table (D10): for each 32-prefix chunk, digit i and
    // value v <= hi_i, the bits of the chunk's prefixes s' with s'_i <= v, at
    // word chunk * TS + dbase[i] + v.  TS = sum_i (hi_i + 1); 0 = no table.
    int32_t TS;
    int32_t hi[MAXK];
    int32_t dbase[MAXK];
    const uint32_t *domtab;     // device table (TS > 0)
    // pivot blocks (D13): blk[2q], blk[2q+1] = [first, end) of the
    // prefixes (indices into the nonzero-prefix list, entry 1 of the prefix
    // table = index 0) whose first nonzero leading digit is q; written by
    // build_prefix_kernel.  A row p != 0 walks only the block of its own first
    // nonzero digit.  Empty block: first == end.
    int32_t *blk;               // device [2 * MAXK]
    // level window (D15): OR-ed into every row's packed digits (the
    // slab digit p0 of a slab launch whose row index holds the p0 = 0 rows), and
    // the word span the kernel may address relative to the table pointer
    // (int32 word offsets; 0 = the whole table)
    uint64_t pw_or[MAXW];
    int64_t span_words;
};
constexpr int64_t DOMTAB_MAX_BYTES = 16384;

// Rows per shard of a sharded row-level: ceil(R / G)
// rounded up so that every shard's compact slice (rows of row_bytes bytes)
// starts 16-byte aligned -- the packed fill kernel writes compact rows with
// vector stores.  Rank g owns rows [g * chunk, min(R, (g + 1) * chunk)); trailing
// ranks may be empty.  Exported as ptas_level_shard.
inline int64_t shard_chunk(int64_t R, int G, int64_t row_bytes)
{
    const int64_t c = (R + G - 1) / G;
    int64_t q = 1;
    while ((q * row_bytes) % 16 != 0) ++q;      // smallest q with q * row_bytes = 0 (mod 16), q <= 16
    return (c + q - 1) / q * q;
}

// Padded row pitch in 32-bit words for a row of `bytes` bytes: a multiple of
// the packed fill kernel's words per lane (2 up to 64 words, 4 up to 128, 8
// beyond), so each lane's chunk is one aligned vector load.
inline int64_t row_pitch_words(int64_t bytes)
{
    const int64_t w = (bytes + 3) / 4;
    const int64_t ch = w < 8 ? 1 : (w <= 64 ? 2 : (w <= 128 ? 4 : 8));
    return (w + ch - 1) / ch * ch;
}

// Dataflow wavefront (one launch for a run of row-levels rho0 .. rho0+nlev-1,
// DESIGN.md D7): warps take row sets in level order from a ticket counter and
// wait only for the ready flags of each row's unit predecessors p - e_i.
// Row sets never straddle a level (a set never waits on itself).
struct DfArgs {
    const int32_t *plan;          // device: [nlev+1] first set of each level, then [nlev+1] first slot
    uint32_t *flags;              // device: one ready flag per row (row-major row id)
    unsigned long long *ticket;   // device: monotone ticket counter of the slot
    unsigned long long base;      // ticket value of set 0 of this launch
    int64_t total_sets;
    int32_t nlev;
    uint32_t epoch;               // flag value meaning "row done in this launch"
    int32_t nsplit;               // 1: one row set per warp; 8: per block (the warps split the prefix walk)
    int32_t grid_div;             // >1: concurrent DPs, the launch takes 1/grid_div of the resident blocks
    int32_t sleep0, sleep_max;    // flag-poll backoff (ns): first sleep, cap
    unsigned long long *prof;     // diagnostics build (PTAS_DF_PROFILE): 6 counters per level, else null
    int32_t rstride[MAXK];        // rows between p and p - e_i (leading digit i)
    uint64_t dmask[MAXK];         // bits of leading digit i inside its packed word g.word[i]
};

// Narrow K = 3 DPs on one thread-block cluster (row_ring.cu, D14).
struct RingArgs {
    int32_t N0, N1;       // the two leading counts (row (a, b), level a + b)
    int64_t stride0;      // elements between rows (a, b) and (a + 1, b)
    int32_t Wp;           // row pitch (elements)
    int32_t Lw, Lg;       // words per row, lanes per row (Lw / CH)
    int32_t J0;           // min(N_last, floor(T / r_last))
    int32_t R;            // ring slots (row-levels resident): Rdep + TB - 1
    int32_t Rdep;         // dependency depth: 1 + the largest leading-digit sum of a configuration
    int32_t A;            // own rows per level per CTA: ceil((N0 + 1) / cluster size)
    int32_t H;            // rows per level below the block a row can read (H = max s0 <= A)
    int32_t TB;           // row-levels per cluster barrier; the halo holds TB * H rows per level
    int32_t rho_max;      // N0 + N1
};

// Device-side summary written by the planning kernels and read back once.
struct DpMeta {
    int64_t nC;            // |C|
    int64_t nP;            // number of prefix entries (incl. the zero prefix)
    unsigned long long relax;  // closed-form relaxations sum_{s in C} prod(N_i - s_i + 1)
    unsigned long long relax_exec;  // (n, s') window gathers of the fill kernels (readings D5, D12,
                                    // D13): sum over prefixes s' != 0 with first nonzero digit q of
                                    // prod_{q<=i<K-1}(N_i - s'_i + 1) * W  (rows p >= s' whose own
                                    // first nonzero digit is q); row p = 0 is a closed form
    int32_t opt;           // OPT(N)
    int32_t err;           // device-detected error (traceback)
    int32_t ovf;           // enumeration without a host round trip: |C| or the prefix
                           // list exceeded the preallocated bounds (the fill kernels
                           // then do nothing and the host redoes the DP synchronously)
    int32_t pad_;
};

// Prefix-list bound of a DP enumerated without a host round trip (= the
// constant bank's CP_MAX): shared-memory tables are sized for it.
constexpr int64_t NP_CAP = 1000;
// Heuristic hint for the fill launchers (prefix-list length estimate of the
// calling DP slot's thread; -1 = use the bound they are given).
extern thread_local int64_t tl_np_hint;

// Prefixes of the pivot-0 block (D13) of a DP in internal class order: #{s' over
// the K - 1 leading classes : s'_0 >= 1, s'_i <= N_i, sum s'_i r_i <= T}, capped
// at `cap` (host; a few microseconds).  Most rows of a DP walk this block.
inline int64_t pivot0_block(const int32_t *N, const int64_t *r, int K, int64_t T, int64_t cap = 4096)
{
    if (K < 2) return 0;
    int64_t cnt = 0;
    // iterative DFS over the leading digits (d[i] = digit i, rem[i] = budget left before digit i)
    int64_t d[64], rem[65];
    const int L = K - 1 < 64 ? K - 1 : 64;
    int i = 0;
    d[0] = 1;
    rem[0] = T;
    if (N[0] < 1 || r[0] > T) return 0;
    for (;;) {
        if (i == L) {   // a complete prefix
            if (++cnt > cap) return cnt;
            --i;
            ++d[i];
            continue;
        }
        if (d[i] <= N[i] && d[i] * r[i] <= rem[i]) {
            rem[i + 1] = rem[i] - d[i] * r[i];
            ++i;
            if (i < L) d[i] = 0;
            continue;
        }
        if (i == 0) return cnt;
        --i;
        ++d[i];
    }
}

// Slab/halo pipeline plan: S slabs of the first
// internal class over `world` ranks; rank `rank` owns [pb, pe), holds [pbase, pe)
// (hin = pb - pbase halo slabs received from rank - 1 per chunk) and sends its
// last hout slabs to rank + 1.  hin of rank g equals hout of rank g - 1.
inline void slab_plan(int64_t S, int64_t hi0, int rank, int world, int64_t *pb, int64_t *pe, int64_t *pbase,
                      int64_t *hin, int64_t *hout)
{
    *pb = S * rank / world;
    *pe = S * (rank + 1) / world;
    *pbase = *pb - hi0 > 0 ? *pb - hi0 : 0;
    *hin = *pb - *pbase;
    *hout = hi0 < *pe ? hi0 : *pe;
}

// ---------------------------------------------------------------- launchers
// All launchers enqueue on `st` and return cudaGetLastError().
// pass 1 writes nothing when the total |C| (offsets[nprefix]) exceeds cap
cudaError_t launch_enum_configs(int pass, int K, int D, int64_t nprefix,
                                const int32_t *hi, const int64_t *r, int64_t T,
                                const int64_t *stride, int64_t *d_counts,
                                const int64_t *d_offsets, uint16_t *d_digits,
                                int64_t *d_off, cudaStream_t st, int64_t cap = INT64_MAX);
cudaError_t launch_exclusive_scan(const int64_t *d_in, int64_t *d_out, int64_t n,
                                  int64_t *d_total, cudaStream_t st);
// Dominance table of the DP's prefixes (g.TS > 0; exits when meta->ovf).
cudaError_t launch_build_dom_table(const PrefixEntry *d_pref, const DpMeta *d_meta, const RowGeom &g,
                                   uint32_t *d_tab, cudaStream_t st);
// |C| = *d_nC (device); nc_cap / np_cap: bounds of the buffers / of the fill
// kernels' prefix tables (exceeded: meta->ovf = 1 and nothing else is written)
cudaError_t launch_build_prefix(int K, const uint16_t *d_digits, const int64_t *d_off,
                                const int64_t *d_nC, int64_t nc_cap, int64_t np_cap, const RowGeom &g,
                                const int32_t *Nall, PrefixEntry *d_pref, DpMeta *d_meta, cudaStream_t st);
// One row-level of the level fill.  e = 1 or 2.  Rows [slot_begin, slot_begin+slot_count)
// of row-level rho; results go to the table (compact_out == NULL) or to
// compact_out[(slot - slot_begin) * Wp + x].
// rb/pw point at the row-level's first slot (rb + level_start[rho]); pw_stride
// is the distance between the packed words of one row (= total rows).
cudaError_t launch_row_fill(int e, void *table, const RowGeom &g, const int64_t *rb,
                            const uint64_t *pw, int64_t pw_stride,
                            const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound,
                            int J0, int rho, int64_t slot_begin, int64_t slot_count,
                            void *compact_out, int sm_count, cudaStream_t st);
// Rows longer than the packed kernel takes (> 1 KiB): cross-row window minima
// (one warp per 32-entry chunk) then the in-row chain (one warp per row).
// Table output only (no compact slices); slot_begin/slot_count as above, rb/pw
// at the row-level's first slot.
cudaError_t launch_row_fill_long(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                 int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 int sm_count, cudaStream_t st);
// a-4 level-ordered row index: for every row slot t (row-levels concatenated,
// lexicographic within a level) its row base index rb[t] and packed leading
// digits pw[w * rows + t].
cudaError_t launch_build_row_index(const RowGeom &g, const int64_t *d_cnt, const int64_t *d_level_start,
                                   int64_t rows, int64_t *d_rb, uint64_t *d_pw, cudaStream_t st);
// Packed-word fill (row_fill_swar.cu); cudaErrorNotSupported -> use launch_row_fill.
// pdl = 1: programmatic dependent launch after the previous fill launch (the
// first fill launch of a DP must use pdl = 0).
cudaError_t launch_row_fill_swar(int e, void *table, const RowGeom &g, const int64_t *rb,
                                 const uint64_t *pw, int64_t pw_stride,
                                 const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound,
                                 int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 void *compact_out, int sm_count, cudaStream_t st, int pdl,
                                 int cslot);
// Dataflow launch over a run of row-levels (D7).  rb/pw are the
// DP's whole row index (slot 0 = row-level 0).  rows_per_set: see
// swar_df_rows_per_set.  *ticket_base advances by the ticket grabs of the
// launch.  cudaErrorNotSupported -> fill the run level by level instead.
cudaError_t launch_row_fill_swar_df(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                    int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                    int64_t nP_bound, int J0, int64_t max_level_rows, const DfArgs &df,
                                    unsigned long long *ticket_base, int sm_count, cudaStream_t st, int pdl,
                                    int cslot);
// Whole level fill of a K = 3 DP on one thread-block cluster with the recent
// row-levels in distributed shared memory (row_ring.cu); N, r internal order.
// cudaErrorNotSupported: the DP does not qualify (use the other launchers);
// dry = true: only the check, no launch.
cudaError_t launch_row_fill_ring(int e, void *table, const RowGeom &g, const int32_t *N, const int64_t *r,
                                 int64_t T, int J0, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, cudaStream_t st, bool dry);
// The paper's Alg 4 / Alg 5 partitioned DP as an A/B baseline (alg4.cu):
// blocked layout, block-levels, in-block levels, full Eq. 1 relaxation per entry.
int alg4_fill(int e, const int32_t *N, int K, const int32_t *cfg_digits, int64_t nC, int dim, void *host_out,
              int32_t *opt_out, double *fill_s, int64_t *nblocks_out, int32_t *block_levels_out, int32_t *div_out);
// Host-only geometry test of launch_row_fill_ring (internal class order).
bool ring_fits(const int32_t *N, const int64_t *r, int K, int64_t T);
// Rows per row set the dataflow kernel will use for this geometry (0 = unsupported).
int swar_df_rows_per_set(int e, const RowGeom &g, int J0, int64_t max_level_rows, int sm_count);
// Copies the DP's prefix offsets/Jmax into the fill kernel's constant bank
// (after build_prefix, before the fill loop); cudaErrorNotSupported when the
// prefix list is too long (the kernels then read it from shared memory).
cudaError_t prepare_const_prefix(const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound, int e,
                                 int nwords, int cslot, void *d_staging, cudaStream_t st);
size_t const_prefix_staging_bytes();
// Traceback with the canonical ranks computed on the device and the machines'
// configurations written in canonical class order (d_out_dig[max_out][Kc]);
// cudaErrorNotSupported when the configurations do not fit shared memory.
cudaError_t launch_traceback_canon(int e, const void *table, int K, const int32_t *d_N, const uint16_t *d_digits,
                                   const int64_t *d_off, int32_t *d_rank, int64_t nC, const int32_t *d_inv, int Kc,
                                   int64_t idx_start, int32_t *d_out, int32_t *d_out_dig, int32_t max_out,
                                   int32_t *d_len, DpMeta *d_meta, cudaStream_t st);
// Copy rows of pitch Wp (src) to pitch W (dst), `rows` rows of e-byte entries.
cudaError_t launch_compact_rows(int e, const void *src, void *dst, int64_t rows, int64_t W,
                                int64_t Wp, cudaStream_t st);
cudaError_t launch_row_scatter(int e, void *table, const RowGeom &g, const int64_t *rb,
                               int64_t slot_count, const void *compact, int sm_count, cudaStream_t st);
cudaError_t launch_row_gather(int e, const void *table, const RowGeom &g, const int64_t *rb, int64_t slot_count,
                              void *compact, int sm_count, cudaStream_t st);
cudaError_t launch_read_opt(int e, const void *table, int64_t idx, DpMeta *d_meta,
                            cudaStream_t st);
cudaError_t launch_traceback(int e, const void *table, int K, const int32_t *d_N,
                             const int64_t *d_stride, const uint16_t *d_digits,
                             const int64_t *d_off, const int32_t *d_rank, int64_t nC,
                             int64_t idx_start, int32_t *d_out, int32_t max_out,
                             int32_t *d_len, DpMeta *d_meta, cudaStream_t st);
cudaError_t launch_fill_value(void *p, int64_t bytes, int value, cudaStream_t st);

}  // namespace ptas
