// obj_easom.cu — instantiates the fused kernels for fastpso::Easom (one TU per
// objective so the library builds in parallel).
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_easom() {
  static const KernelTable t = make_kernel_table<Easom>();
  return &t;
}
}  // namespace fastpso
