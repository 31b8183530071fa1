// obj_user.cu — instantiates the fused kernels for every user functor listed
// in PSO_USER_OBJECTIVES (user_objectives.cuh), the paper's customisation
// schema (Sec 3.2) at compile time.
#include "swarm_kernels.cuh"

namespace fastpso {
const KernelTable* kernels_user(int objective) {
#define PSO_CASE(ID, F)                                     \
  case ID: {                                                \
    static const KernelTable t = make_kernel_table<F>();    \
    return &t;                                              \
  }
  switch (objective) {
    PSO_USER_OBJECTIVES(PSO_CASE)
    default:
      return nullptr;
  }
#undef PSO_CASE
}
}  // namespace fastpso
