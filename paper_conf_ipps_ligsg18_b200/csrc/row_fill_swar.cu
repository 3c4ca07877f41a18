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

#include "internal.h"

namespace ptas {

#define PTAS_SWAR_DECL(tag)                                                                          \
    cudaError_t launch_row_fill_swar_##tag(int e, void *table, const RowGeom &g, const int64_t *rb,      \
                                           const uint64_t *pw, int64_t pw_stride,                        \
                                           const PrefixEntry *d_pref, const DpMeta *d_meta,               \
                                           int64_t nP_bound, int J0, int rho, int64_t slot_begin,         \
                                           int64_t slot_count, void *compact_out, int sm_count,           \
                                           cudaStream_t st, int pdl, int cslot);                       \
    cudaError_t prepare_const_prefix_##tag(const PrefixEntry *d_pref, const DpMeta *d_meta,             \
                                           int64_t nP_bound, int e, int cslot, void *d_staging, cudaStream_t st);
PTAS_SWAR_DECL(u8_nw1)
PTAS_SWAR_DECL(u8_nw2)
PTAS_SWAR_DECL(u16_nw1)
PTAS_SWAR_DECL(u16_nw2)
#undef PTAS_SWAR_DECL

#define PTAS_SWAR_DF_DECL(tag)                                                                        \
    cudaError_t launch_row_fill_swar_df_##tag(int e, void *table, const RowGeom &g, const int64_t *rb,     \
                                              const uint64_t *pw, int64_t pw_stride,                       \
                                              const PrefixEntry *d_pref, const DpMeta *d_meta,              \
                                              int64_t nP_bound, int J0, int64_t max_level_rows,             \
                                              const DfArgs &df, unsigned long long *ticket_base,            \
                                              int sm_count, cudaStream_t st, int pdl, int cslot);
PTAS_SWAR_DF_DECL(u8_nw1)
PTAS_SWAR_DF_DECL(u8_nw2)
PTAS_SWAR_DF_DECL(u16_nw1)
PTAS_SWAR_DF_DECL(u16_nw2)
#undef PTAS_SWAR_DF_DECL

cudaError_t launch_row_fill_swar(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                 int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 void *compact_out, int sm_count, cudaStream_t st, int pdl, int cslot)
{
    const bool two = g.nwords > 1;
#define PTAS_SWAR_CALL(tag)                                                                             \
    return launch_row_fill_swar_##tag(e, table, g, rb, pw, pw_stride, d_pref, d_meta, nP_bound, J0, rho,     \
                                      slot_begin, slot_count, compact_out, sm_count, st, pdl, cslot)
    if (e == 1) {
        if (!two) PTAS_SWAR_CALL(u8_nw1);
        PTAS_SWAR_CALL(u8_nw2);
    }
    if (!two) PTAS_SWAR_CALL(u16_nw1);
    PTAS_SWAR_CALL(u16_nw2);
#undef PTAS_SWAR_CALL
}

cudaError_t launch_row_fill_swar_df(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                    int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                    int64_t nP_bound, int J0, int64_t max_level_rows, const DfArgs &df,
                                    unsigned long long *ticket_base, int sm_count, cudaStream_t st, int pdl,
                                    int cslot)
{
    const bool two = g.nwords > 1;
#define PTAS_SWAR_DF_CALL(tag)                                                                            \
    return launch_row_fill_swar_df_##tag(e, table, g, rb, pw, pw_stride, d_pref, d_meta, nP_bound, J0,     \
                                         max_level_rows, df, ticket_base, sm_count, st, pdl, cslot)
    if (e == 1) {
        if (!two) PTAS_SWAR_DF_CALL(u8_nw1);
        PTAS_SWAR_DF_CALL(u8_nw2);
    }
    if (!two) PTAS_SWAR_DF_CALL(u16_nw1);
    PTAS_SWAR_DF_CALL(u16_nw2);
#undef PTAS_SWAR_DF_CALL
}

cudaError_t prepare_const_prefix(const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound, int e, int nwords,
                                 int cslot, void *d_staging, cudaStream_t st)
{
    const bool two = nwords > 1;
    if (e == 1) return two ? prepare_const_prefix_u8_nw2(d_pref, d_meta, nP_bound, e, cslot, d_staging, st)
                           : prepare_const_prefix_u8_nw1(d_pref, d_meta, nP_bound, e, cslot, d_staging, st);
    return two ? prepare_const_prefix_u16_nw2(d_pref, d_meta, nP_bound, e, cslot, d_staging, st)
               : prepare_const_prefix_u16_nw1(d_pref, d_meta, nP_bound, e, cslot, d_staging, st);
}

size_t const_prefix_staging_bytes() { return 8 + 8 * 1000; }

}  // namespace ptas
