// solver_inst_pbicgstab_1024.cu -- instantiations of pbicgstab_persistent for blocks of <= 1024 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_pbicgstab_1024, pbicgstab_persistent, 1024)
}  // namespace mf
