// obj_griewank.cu — instantiates the fused kernels for fastpso::Griewank (one TU per
// objective so the library builds in parallel).
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_griewank() {
  static const KernelTable t = make_kernel_table<Griewank>();
  return &t;
}
}  // namespace fastpso
