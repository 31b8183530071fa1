// obj_rosenbrock.cu — instantiates the fused kernels for fastpso::Rosenbrock (one TU per
// objective so the library builds in parallel).
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_rosenbrock() {
  static const KernelTable t = make_kernel_table<Rosenbrock>();
  return &t;
}
}  // namespace fastpso
