// precond.cu -- ILU(0) preconditioning.  (filled in below)
#include "mf_internal.cuh"

extern "C" {
mf_status mf_precond_create(const mf_tile_matrix*, mf_precond_kind, mf_stream, mf_precond** out) {
    if (out) *out = nullptr;
    return mf::fail(MF_ERR_NOT_IMPLEMENTED, "ILU(0) not built yet");
}
mf_status mf_precond_destroy(mf_precond*) { return MF_OK; }
mf_status mf_precond_apply(const mf_precond*, const double*, double*, mf_stream) {
    return mf::fail(MF_ERR_NOT_IMPLEMENTED, "ILU(0) not built yet");
}
}
