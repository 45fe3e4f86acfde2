// dist.cu -- row-block multi-GPU solve over NCCL.  (filled in below)
#include "mf_internal.cuh"

extern "C" {
mf_status mf_comm_unique_id(void*) { return mf::fail(MF_ERR_NOT_IMPLEMENTED, "multi-GPU not built yet"); }
mf_status mf_comm_create(const void*, int32_t, int32_t, mf_comm** out) {
    if (out) *out = nullptr;
    return mf::fail(MF_ERR_NOT_IMPLEMENTED, "multi-GPU not built yet");
}
mf_status mf_comm_destroy(mf_comm*) { return MF_OK; }
mf_status mf_tile_matrix_from_csr_dist(mf_comm*, int64_t, int64_t, int64_t, int64_t, const int64_t*, const int32_t*,
                                       const double*, const mf_convert_opts*, mf_stream, mf_tile_matrix** out) {
    if (out) *out = nullptr;
    return mf::fail(MF_ERR_NOT_IMPLEMENTED, "multi-GPU not built yet");
}
mf_status mf_cg_solve_dist(const mf_tile_matrix*, const double*, double*, const mf_solve_opts*, mf_solve_info*,
                           mf_stream) {
    return mf::fail(MF_ERR_NOT_IMPLEMENTED, "multi-GPU not built yet");
}
}
