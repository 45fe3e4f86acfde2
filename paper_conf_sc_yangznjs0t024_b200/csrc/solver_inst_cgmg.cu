// solver_inst_cgmg.cu -- instantiations of the device-initiated multi-GPU CG (cg_persistent with
// the MG hooks: peer halo stores, arrival counters, rank-ordered cross-GPU reductions)
#include "solver_kernels.cuh"

namespace mf {
void* pick_cgmg(int maxt, bool dyn) {
    if (maxt > 512) return dyn ? (void*)cg_persistent<true, false, false, 1024, true> : (void*)cg_persistent<false, false, false, 1024, true>;
    return dyn ? (void*)cg_persistent<true, false, false, 512, true> : (void*)cg_persistent<false, false, false, 512, true>;
}
}  // namespace mf
