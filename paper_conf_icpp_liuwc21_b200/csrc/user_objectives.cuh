// user_objectives.cuh — user-defined objectives, the paper's customisation
// schema (Sec 3.2: "lambda(.) is the function that practitioners
// can implement by themselves and pass to FastPSO").
//
// To add an objective: write a functor with the interface documented in
// objectives.cuh, append X(<id>, <Functor>) to PSO_USER_OBJECTIVES with an id
// >= PSO_OBJ_CUSTOM_BASE (64), and rebuild (`make lib`).  The fused kernel is
// instantiated for it at compile time: no JIT, no Triton, no CPU fallback.
//
// Ackley ships through this path (id PSO_OBJ_ACKLEY = 5) to exercise it.
#pragma once

namespace fastpso {
namespace user {

// Ackley ([20]):
//   f = -20 exp(-0.2 sqrt(S/d)) - exp(C/d) + 20 + e,  S = sum x^2, C = sum cos(2 pi x)
//     = 20 (1 - exp(-0.2 sqrt(S/d))) + e (1 - exp(-2 S2/d)),  S2 = sum sin^2(pi x)
// using C = d - 2 S2.  Both sums have nonnegative terms and both cancelling
// pairs go through expm1, so f(0) = 0 exactly and f is accurate near 0.
struct Ackley {
  static constexpr int kAcc = 2;
  static constexpr bool kNeighbor = false;
  __device__ static void init(float* a) {
    a[0] = 0.f;
    a[1] = 0.f;
  }
  __device__ static void map(float* a, float x, float, int, int) {
    a[0] = fmaf(x, x, a[0]);
    a[1] += sinpi_sq(x);
  }
  __device__ static void combine(float* a, const float* b) {
    a[0] += b[0];
    a[1] += b[1];
  }
  __device__ static float finalize(const float* a, int d) {
    const float inv_d = 1.f / (float)d;
    const float t1 = -20.f * expm1f(-0.2f * sqrtf(a[0] * inv_d));
    const float t2 = -2.718281828459045f * expm1f(-2.f * a[1] * inv_d);
    return t1 + t2;
  }
};

}  // namespace user
}  // namespace fastpso

#define PSO_USER_OBJECTIVES(X) X(5, ::fastpso::user::Ackley)
