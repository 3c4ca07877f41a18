// row_fill_swar_u8_nw2.cu — instantiation unit of the packed-word fill kernel (uint8_t, 2 digit word(s)).
#include "row_fill_swar.cuh"

namespace ptas {

cudaError_t launch_row_fill_swar_u8_nw2(int e, void *table, const RowGeom &g, const int64_t *rb, const uint64_t *pw,
                                 int64_t pw_stride, const PrefixEntry *d_pref, const DpMeta *d_meta,
                                 int64_t nP_bound, int J0, int rho, int64_t slot_begin, int64_t slot_count,
                                 void *compact_out, int sm_count, cudaStream_t st, int pdl, int cslot)
{
    return swar::launch_swar_impl<uint8_t, 2>(e, table, g, rb, pw, pw_stride, d_pref, d_meta, nP_bound, J0, rho,
                                          slot_begin, slot_count, compact_out, sm_count, st, pdl, cslot);
}

cudaError_t prepare_const_prefix_u8_nw2(const PrefixEntry *d_pref, const DpMeta *d_meta, int64_t nP_bound, int e,
                                  int cslot, void *d_staging, cudaStream_t st)
{
    return swar::prepare_const_prefix_tu(d_pref, d_meta, nP_bound, e, cslot, d_staging, st);
}

cudaError_t launch_row_fill_swar_df_u8_nw2(int e, void *table, const RowGeom &g, const int64_t *rb,
                                    const uint64_t *pw, int64_t pw_stride, const PrefixEntry *d_pref,
                                    const DpMeta *d_meta, int64_t nP_bound, int J0, int64_t max_level_rows,
                                    const DfArgs &df, unsigned long long *ticket_base, int sm_count,
                                    cudaStream_t st, int pdl, int cslot)
{
    return swar::launch_swar_df_impl<uint8_t, 2>(e, table, g, rb, pw, pw_stride, d_pref, d_meta, nP_bound, J0,
                                              max_level_rows, df, ticket_base, sm_count, st, pdl, cslot);
}

}  // namespace ptas
