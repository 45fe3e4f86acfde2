// solver_inst_pbicgstab_512.cu -- instantiations of pbicgstab_persistent for blocks of <= 512 threads
// (one translation unit per kernel family: the build compiles them in parallel)
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_pbicgstab_512, pbicgstab_persistent, 512)
}  // namespace mf
