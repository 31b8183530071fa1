// objectives.cuh — compile-time objective functors (the paper's user-defined
// evaluation schema, Sec 3.2, without an extended lambda or a JIT).
//
// A functor F describes a per-particle fitness as map -> reduce -> finalize
// over the particle's d coordinates, so it can be fused into the swarm-update
// kernel: each thread maps the coordinates it just updated into kAcc fp32
// accumulators, the CTA tree-reduces them with F::combine, and one thread
// calls F::finalize.  Interface:
//
//   static constexpr int  kAcc;        // accumulators per thread (1 or 2)
//   static constexpr bool kNeighbor;   // map() needs x_{j+1} (Rosenbrock)
//   __device__ static void  init(float* a);                 // identities
//   __device__ static void  map(float* a, float x, float xnext, int j, int d);
//                                      // j: 0-based dim; xnext valid iff kNeighbor && j+1 < d
//   __device__ static void  combine(float* a, const float* b);   // associative
//   __device__ static float finalize(const float* a, int d);
//   optional:
//   __device__ static void  map4(float* a, float4 x, float xnext, int j, int d);
//                                      // == map over dims j..j+3 (all < d), same bits
//   static constexpr bool kRowTable;   // with table4 / map4r: per-dimension factors
//   __device__ static float4 table4(int j);          // computed once per kernel (the
//   __device__ static void  map4r(float* a, float4 x, int d, const float4& t);
//                                      // TMA kernel's threads own fixed dims); map4r
//                                      // with t = table4(j) == map4 at j, same bits
//
// The reduction order is fixed by the launch shape, which depends only on d,
// so fitness bits do not depend on the grid or on the number of GPUs.
// Formulas are rearranged for fp32 accuracy where that is free (noted below);
// all are mathematically the definitions in include/fastpso.h.
#pragma once

namespace fastpso {

// sin^2(pi x) for any finite fp32 x, <= ~4 ulp relative: r = x - rint(x) is
// exact (|r| <= 1/2) and sin^2(pi r) = u P(u), u = r^2, with a degree-5
// least-squares fit of sin^2(pi sqrt(u)) / u on [0, 1/4] (approximation error
// 1.4e-8 relative; fp32 Horner evaluation <= 3.2 ulp, checked exhaustively on a
// 4e5-point grid).  Shared by the periodic objectives:
//   10 - 10 cos(2 pi x) = 20 sin^2(pi x),   cos(y) = 1 - 2 sin^2(pi y / (2 pi)).
__device__ __forceinline__ float sinpi_sq(float x) {
  const float r = x - rintf(x);
  const float u = r * r;
  float p = -3.335728645324707f;
  p = fmaf(p, u, 13.036796569824219f);
  p = fmaf(p, u, -30.098480224609375f);
  p = fmaf(p, u, 42.72692108154297f);
  p = fmaf(p, u, -32.469661712646484f);
  p = fmaf(p, u, 9.869604110717773f);
  return u * p;
}

// 20 sin^2(pi x), the Rastrigin term, with the 20 folded into the coefficients
// of sinpi_sq (each rounded once to fp32): one multiply less per element,
// <= 4 ulp relative (checked on a 4e5-point grid over r in [-1/2, 1/2]).
__device__ __forceinline__ float sinpi_sq20(float x) {
  const float r = x - rintf(x);
  const float u = r * r;
  float p = -66.71456909179688f;
  p = fmaf(p, u, 260.7359313964844f);
  p = fmaf(p, u, -601.9696044921875f);
  p = fmaf(p, u, 854.5384521484375f);
  p = fmaf(p, u, -649.3932495117188f);
  p = fmaf(p, u, 197.39208984375f);
  return u * p;
}

constexpr float kInv2Pi = 0.15915494309189535f;

// Sphere: sum x_k^2.
struct Sphere {
  static constexpr int kAcc = 1;
  static constexpr bool kNeighbor = false;
  __device__ static void init(float* a) { a[0] = 0.f; }
  __device__ static void map(float* a, float x, float, int, int) { a[0] = fmaf(x, x, a[0]); }
  __device__ static void combine(float* a, const float* b) { a[0] += b[0]; }
  __device__ static float finalize(const float* a, int) { return a[0]; }
};

// Rastrigin ([20]): sum x^2 + 10 - 10 cos(2 pi x) = sum x^2 + 20 sin^2(pi x).
// The sin^2 form has no cancellation, so every term is computed to a few ulp.
struct Rastrigin {
  static constexpr int kAcc = 1;
  static constexpr bool kNeighbor = false;
  __device__ static void init(float* a) { a[0] = 0.f; }
  __device__ static void map(float* a, float x, float, int, int) {
    a[0] += fmaf(x, x, sinpi_sq20(x));
  }
  __device__ static void combine(float* a, const float* b) { a[0] += b[0]; }
  __device__ static float finalize(const float* a, int) { return a[0]; }
};

// Rosenbrock ([20]): sum_{k<d} 100 (x_{k+1} - x_k^2)^2 + (x_k - 1)^2.
struct Rosenbrock {
  static constexpr int kAcc = 1;
  static constexpr bool kNeighbor = true;
  __device__ static void init(float* a) { a[0] = 0.f; }
  __device__ static void map(float* a, float x, float xn, int j, int d) {
    if (j + 1 < d) {
      const float t = fmaf(-x, x, xn);
      const float u = x - 1.f;
      a[0] += fmaf(100.f * t, t, u * u);
    }
  }
  __device__ static void combine(float* a, const float* b) { a[0] += b[0]; }
  __device__ static float finalize(const float* a, int) { return a[0]; }
};

// Griewank: 1 + sum x_k^2 / 4000 - prod cos(x_k / sqrt(k)), k = j + 1.
struct Griewank {
  static constexpr int kAcc = 2;
  static constexpr bool kNeighbor = false;
  __device__ static void init(float* a) {
    a[0] = 0.f;
    a[1] = 1.f;
  }
  // k = j + 1 >= 1 is never subnormal, so the flush-to-zero MUFU form is
  // bitwise rsqrtf (whose non-FTZ form adds a subnormal-input rescale).
  __device__ static float rsqrt_k(float k) {
    float r;
    asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(k));
    return r;
  }
  __device__ static void term_r(float* a, float x, float r) {  // r = rsqrt_k(k)
    a[0] = fmaf(x, x, a[0]);
    const float y = x * r;  // x_k / sqrt(k)
    a[1] *= fmaf(-2.f, sinpi_sq(y * kInv2Pi), 1.f);  // cos(y)
  }
  __device__ static void term(float* a, float x, float k) { term_r(a, x, rsqrt_k(k)); }
  // Row-invariant per-dimension factors: a streaming kernel whose threads own
  // the same dims in every row computes rsqrt(k) once per kernel (table4) and
  // maps with them (map4r) -- the same bits as map4, one MUFU + one add fewer
  // per element.
  static constexpr bool kRowTable = true;
  __device__ static float4 table4(int j) {
    const float k = (float)(j + 1);
    return make_float4(rsqrt_k(k), rsqrt_k(k + 1.f), rsqrt_k(k + 2.f), rsqrt_k(k + 3.f));
  }
  __device__ static void map4r(float* a, float4 x, int, const float4& r) {
    term_r(a, x.x, r.x);
    term_r(a, x.y, r.y);
    term_r(a, x.z, r.z);
    term_r(a, x.w, r.w);
  }
  __device__ static void map(float* a, float x, float, int j, int) { term(a, x, (float)(j + 1)); }
  // Four consecutive dims j..j+3 (j + 4 <= d <= 2^24): (float)(j + 1 + m) ==
  // (float)(j + 1) + m exactly, one conversion instead of four; same bits as map.
  __device__ static void map4(float* a, float4 x, float, int j, int) {
    const float k = (float)(j + 1);
    term(a, x.x, k);
    term(a, x.y, k + 1.f);
    term(a, x.z, k + 2.f);
    term(a, x.w, k + 3.f);
  }
  __device__ static void combine(float* a, const float* b) {
    a[0] += b[0];
    a[1] *= b[1];
  }
  __device__ static float finalize(const float* a, int) {
    return a[0] * (1.f / 4000.f) + (1.f - a[1]);
  }
};

// Easom: -(-1)^d prod cos^2(x_k) exp(-sum (x_k - pi)^2).
struct Easom {
  static constexpr int kAcc = 2;
  static constexpr bool kNeighbor = false;
  __device__ static void init(float* a) {
    a[0] = 1.f;
    a[1] = 0.f;
  }
  __device__ static void map(float* a, float x, float, int, int) {
    const float c = cosf(x);  // accurate near its zeros (cos^2 is relative here)
    const float e = x - 3.14159265358979f;
    a[0] *= c * c;
    a[1] = fmaf(e, e, a[1]);
  }
  __device__ static void combine(float* a, const float* b) {
    a[0] *= b[0];
    a[1] += b[1];
  }
  __device__ static float finalize(const float* a, int d) {
    const float v = a[0] * expf(-a[1]);
    return (d & 1) ? v : -v;
  }
};

}  // namespace fastpso

#include "user_objectives.cuh"

// Built-in objective registry: X(id, Functor).  User functors are listed in
// PSO_USER_OBJECTIVES (user_objectives.cuh).
#define PSO_BUILTIN_OBJECTIVES(X)     \
  X(1, ::fastpso::Sphere)             \
  X(2, ::fastpso::Rastrigin)          \
  X(3, ::fastpso::Rosenbrock)         \
  X(4, ::fastpso::Griewank)           \
  X(6, ::fastpso::Easom)

#define PSO_ALL_OBJECTIVES(X) PSO_BUILTIN_OBJECTIVES(X) PSO_USER_OBJECTIVES(X)
