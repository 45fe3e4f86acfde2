// solver_inst_cgsr_1024.cu -- instantiations of cgsr_persistent (single-reduction CG) for blocks of <= 1024 threads
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_cgsr_1024, cgsr_persistent, 1024)
}  // namespace mf
