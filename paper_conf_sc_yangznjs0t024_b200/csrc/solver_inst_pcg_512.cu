// solver_inst_pcg_512.cu -- instantiations of pcg_persistent for blocks of <= 512 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_pcg_512, pcg_persistent, 512)
}  // namespace mf
