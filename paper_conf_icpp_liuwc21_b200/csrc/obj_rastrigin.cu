// obj_rastrigin.cu — instantiates the fused kernels for fastpso::Rastrigin (one TU per
// objective so the library builds in parallel).
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_rastrigin() {
  static const KernelTable t = make_kernel_table<Rastrigin>();
  return &t;
}
}  // namespace fastpso
