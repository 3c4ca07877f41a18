// row_fill_swar.cu — packed-word level fill, the production kernel of §8(a) a-5
// (dispatch by entry type and digit words; the kernel template is in
// row_fill_swar.cuh, its instantiations in row_fill_swar_<E>_nw<NW>.cu).
//
// Eq. 1 of PAPER.md:74-79 on the row wavefront (D1): a lane group
// owns a row p, each lane CH 32-bit words of it (4 uint8 or 2 uint16 states
// per word; rows padded to a multiple of CH words, D3).  For every prefix s'
// of the row's pivot block (D13) with s' <= p the lanes take ONE vector load
// of the source row p - s' and ONE shifted window of it (the clamp
// x - min(x, Jmax(s')) of D5, built from the left neighbour's words by shuffles
// and a PRMT; uint8 as even/odd uint16 lanes with the sign-replicating PRMT, a
// monotone encoding), and keep the minimum with VIMNMX.U16x2.  The row is then
// 1 + that minimum (D12: the in-row configurations never win for p != 0; row 0
// is ceil(x / J0)); there is no in-row closure and no chain.  Each (row,
// prefix, x) is evaluated once; the executed count is stats.relax_executed.
// Entries in the row padding are computed but never read as sources.
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
