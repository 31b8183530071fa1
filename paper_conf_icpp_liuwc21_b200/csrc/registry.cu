// registry.cu — objective id -> kernel table (built-ins: include/fastpso.h
// PSO_OBJ_*; user functors: user_objectives.cuh).
#include "kernels.h"

namespace fastpso {
const KernelTable* kernels_sphere();
const KernelTable* kernels_rastrigin();
const KernelTable* kernels_rosenbrock();
const KernelTable* kernels_griewank();
const KernelTable* kernels_easom();
const KernelTable* kernels_user(int objective);

const KernelTable* kernel_table(int objective) {
  switch (objective) {
    case 1: return kernels_sphere();
    case 2: return kernels_rastrigin();
    case 3: return kernels_rosenbrock();
    case 4: return kernels_griewank();
    case 6: return kernels_easom();
    default: return kernels_user(objective);
  }
}
}  // namespace fastpso
