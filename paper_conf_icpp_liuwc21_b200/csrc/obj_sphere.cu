// obj_sphere.cu — instantiates the fused kernels for fastpso::Sphere (one TU per
// objective so the library builds in parallel).
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_sphere() {
  static const KernelTable t = make_kernel_table<Sphere>();
  return &t;
}
}  // namespace fastpso
