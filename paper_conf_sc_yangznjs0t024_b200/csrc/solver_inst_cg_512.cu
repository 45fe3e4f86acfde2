// solver_inst_cg_512.cu -- instantiations of cg_persistent for blocks of <= 512 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_cg_512, cg_persistent, 512)
}  // namespace mf
