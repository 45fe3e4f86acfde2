// solver_inst_cgsr_512.cu -- instantiations of cgsr_persistent (single-reduction CG) for blocks of <= 512 threads
#include "solver_kernels.cuh"

namespace mf {
MF_DEFINE_PICK(pick_cgsr_512, cgsr_persistent, 512)
}  // namespace mf
