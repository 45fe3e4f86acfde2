// solver_inst_bicgstab_1024.cu -- instantiations of bicgstab_persistent for blocks of <= 1024 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_bicgstab_1024, bicgstab_persistent, 1024)
}  // namespace mf
