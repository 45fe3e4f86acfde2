// solver_inst_cg_1024.cu -- instantiations of cg_persistent for blocks of <= 1024 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_cg_1024, cg_persistent, 1024)
}  // namespace mf
