// solver_inst_pcg_1024.cu -- instantiations of pcg_persistent for blocks of <= 1024 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_pcg_1024, pcg_persistent, 1024)
}  // namespace mf
