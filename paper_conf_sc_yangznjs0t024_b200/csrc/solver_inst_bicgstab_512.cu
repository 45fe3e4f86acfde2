// solver_inst_bicgstab_512.cu -- instantiations of bicgstab_persistent for blocks of <= 512 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_bicgstab_512, bicgstab_persistent, 512)
}  // namespace mf
