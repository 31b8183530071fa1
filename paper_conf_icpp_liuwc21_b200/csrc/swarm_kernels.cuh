// swarm_kernels.cuh — the fused FastPSO iteration for sm_100a (kernel templates).
//
// Instantiated once per objective functor in obj_*.cu (parallel build); the
// host side (planning, launches, the gbest rebest/select kernels) is
// swarm_host.cu.
//
// One kernel per iteration replaces the paper's five phases (Fig. 5, P:L561-567:
// init / eval / pbest / gbest / swarm) and its materialised random matrices.
// Per particle row (one CTA per row at a time, persistent grid):
//
//   A1  r1, r2 = Philox4x32-10(seed, t, i, q) in registers        (Eq. 1 l, g)
//   A2  v' = (w v + (c1 r1)(pb - x)) + (c2 r2)(g - x)              (Eq. 1/4)
//   A3  v' = clamp(v', -vmax, vmax)                                (Eq. 5)
//   A4  x' = clamp(x + v', lo, hi)                                 (Eq. 2; reading 2)
//   A5  f = F(x') : functor map + warp shuffle + CTA tree          (Sec 3.2)
//   A6  if f < pf: pf = f, PB row = x'  (strict)                   (Sec 3.3)
//   A7  gbest: block min of (ord(f), i) over rows with f < gf      (Sec 3.3)
//       -> atomicMin(u64) -> the last CTA copies PB[gi] -> G
//
// HBM traffic per particle-dim update: 12 B read (x, v, pb) + 8 B written
// (x, v) + 4 rho B (pbest copy) + (4 + 4 rho)/d (pf).  G (4 d B) is staged
// into shared memory once per CTA per iteration by a bulk async copy (TMA
// engine, cp.async.bulk + mbarrier) and read from there for every row.
//
// Two variants of the step kernel share the row arithmetic:
//   k_step_tma  (rows of >= 256 dims): warp-specialised.  One producer warp
//               streams whole x / v / pb rows into a ring of shared-memory
//               stages with cp.async.bulk (TMA engine) and mbarrier
//               complete_tx; the compute warps drain the ring.  Memory-level
//               parallelism is the ring depth, independent of registers.
//   k_step_reg  (short rows): every thread loads its float4s with 128-bit
//               LDGs; many rows per SM in flight through occupancy.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <type_traits>

#include "kernels.h"
#include "objectives.cuh"
#include "philox.cuh"

// The row-invariant Philox rounds in the 256-thread instantiation as well (scalar
// bounds only; the per-dimension-bounds variants would pass 88 registers).
// Round 2, A/B of two builds on one box: C4 526.6 -> 523.9 us, NS 642.9 -> 641.0 us
// (round 1 had measured NS +0.8 % with an earlier version of the kernel).
#ifndef PSO_SLOT_PHILOX_NARROW
#define PSO_SLOT_PHILOX_NARROW 1
#endif
#ifndef PSO_SLOT_PHILOX
#define PSO_SLOT_PHILOX 1
#endif

namespace fastpso {
namespace {

// Device-side bounds checks (make lib EXTRA=-DPSO_DEVICE_CHECKS): row / tile
// indices, shared-memory extents of the rings and global offsets, checked on
// every item; a failed check prints and traps (poisoning the handle).  Off in
// the product build.  (compute-sanitizer is closed on the GPU pool since the
// end of round 2; this build is the replacement check, tools/device_checks.sh.)
#ifdef PSO_DEVICE_CHECKS
#define PSO_DCHECK(c)                                                                   \
  do {                                                                                 \
    if (!(c)) {                                                                        \
      printf("PSO_DCHECK %s:%d block %d thread %d: %s\n", __FILE__, __LINE__,        \
             (int)blockIdx.x, (int)threadIdx.x, #c);                                   \
      __trap();                                                                        \
    }                                                                                  \
  } while (0)
#else
#define PSO_DCHECK(c) \
  do {                \
  } while (0)
#endif
__device__ __forceinline__ unsigned dyn_smem_bytes() {
  unsigned v;
  asm volatile("mov.u32 %0, %%dynamic_smem_size;" : "=r"(v));
  return v;
}

constexpr int kMaxThreads = 256;         // compute threads per CTA
constexpr int kMaxThreadsCluster = 512;  // compute threads per CTA of the cluster kernel
constexpr int kMaxThreadsWide = 512;     // compute threads per CTA of the wide TMA variant
constexpr int kMaxStages = 8;
// ring stages of the cluster kernel (its static shared arrays are sized by it; a
// 2-CTA cluster's two 96 KB stages fit only with the static part this small)
constexpr int kClusterStages = 4;
constexpr unsigned kFull = 0xFFFFFFFFu;

// ---------------------------------------------------------------- helpers
// Monotone float -> u32 map (ord(a) < ord(b) <=> a < b for non-NaN a, b);
// -0 is canonicalised to +0 (reading 10).
__device__ __forceinline__ uint32_t ord_f32(float f) {
  const uint32_t u = __float_as_uint(f == 0.f ? 0.f : f);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ unsigned long long pack_key(float f, uint32_t gi) {
  return ((unsigned long long)ord_f32(f) << 32) | gi;
}

__device__ __forceinline__ float4 ld_stream(const float4* p) {
  float4 r;
  asm volatile("ld.global.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st_stream(float4* p, float4 v) {
  asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x),
               "f"(v.y), "f"(v.z), "f"(v.w)
               : "memory");
}

// Named barrier 1 over the n compute threads (the producer warp never joins).
__device__ __forceinline__ void team_sync(int n) {
  asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory");
}

// --- programmatic dependent launch (PDL): consecutive step kernels of one
// stream are launched with programmatic stream serialization, so the next
// iteration's grid is scheduled while this one drains; every global read of
// the next kernel sits behind griddepcontrol.wait (the previous grid has
// completed and its writes are visible).  Without the launch attribute both
// are no-ops.
__device__ __forceinline__ void pdl_wait_and_release() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// --- mbarrier + bulk async copy global -> shared (TMA engine) -------------
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count)
               : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
// try_wait with a suspend-time hint: the waiting warp sleeps in hardware until
// the phase completes (or ~1 ms passes) instead of re-polling, which left
// ~25 % of the TMA kernel's issued instructions in wait loops.
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(phase), "r"(1000000u)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes,
                                         unsigned long long* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}

__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, unsigned bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
               "r"(smem_addr(src)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() {
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// Hint: bring [src, src + bytes) into L2 (no shared memory, no completion).
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, unsigned bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() {
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_shared() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// --- thread-block clusters: DSMEM stores and remote mbarrier arrivals -----
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}
// Address of `p` (this CTA's shared memory) in the shared window of CTA `rank`.
__device__ __forceinline__ uint32_t map_to_rank(const void* p, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_addr(p)), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_cluster_f32(uint32_t addr, float v) {
  asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
// Store into another CTA's shared memory and signal its mbarrier (complete_tx).
__device__ __forceinline__ void st_async_v4(uint32_t addr, float4 v, uint32_t bar_addr) {
  asm volatile(
      "st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(addr),
      "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "r"(bar_addr)
      : "memory");
}
__device__ __forceinline__ void st_async_v2(uint32_t addr, float2 v, uint32_t bar_addr) {
  asm volatile(
      "st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.f32 [%0], {%1, %2}, [%3];" ::"r"(addr),
      "f"(v.x), "f"(v.y), "r"(bar_addr)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t bar_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar_addr)
               : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(unsigned long long* bar, unsigned phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAITC_%=:\n"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAITC_%=;\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(phase)
      : "memory");
}

// --- Eq. 1, 5, 2 on one element, fixed fp32 order, no contraction --------
// The oracle computes b = (c1 * r1) * (pb - x) with r1 = m 2^-24 (m the 24-bit
// Philox integer).  Here c1s = c1 2^-24 is folded once per kernel, and
// c1s * m == c1 * r1 bit for bit: scaling by a power of two commutes with
// round-to-nearest while no operand or result is subnormal, which the ABI
// guarantees by accepting only c1, c2 = 0 or |c1|, |c2| >= 2^-100.
struct MoveParams {
  float w, c1s, c2s, lo, hi, vmax;
};
__device__ __forceinline__ MoveParams move_params(const SwarmArgs& a) {
  return MoveParams{a.w, __fmul_rn(a.c1, 0x1p-24f), __fmul_rn(a.c2, 0x1p-24f), a.lo, a.hi, a.vmax};
}
__device__ __forceinline__ void move1(const MoveParams& m, float& x, float& v, float pb, float g,
                                      float m1, float m2) {
  const float a = __fmul_rn(m.w, v);
  const float b = __fmul_rn(__fmul_rn(m.c1s, m1), __fsub_rn(pb, x));
  const float c = __fmul_rn(__fmul_rn(m.c2s, m2), __fsub_rn(g, x));
  float vn = __fadd_rn(__fadd_rn(a, b), c);
  vn = fminf(fmaxf(vn, -m.vmax), m.vmax);
  x = fminf(fmaxf(__fadd_rn(x, vn), m.lo), m.hi);
  v = vn;
}

// Eq. 1 with per-dimension bounds (NEXT-2 reading of Eq. 5):
// v' = clamp(v', vlo_j, vhi_j), x' = clamp(x + v', xlo_j, xhi_j).  With the
// scalar bounds (vlo = -vmax, vhi = vmax, xlo = lo, xhi = hi) this is move1.
__device__ __forceinline__ void move1b(const MoveParams& m, float& x, float& v, float pb, float g,
                                       float m1, float m2, float vlo, float vhi, float xlo,
                                       float xhi) {
  const float a = __fmul_rn(m.w, v);
  const float b = __fmul_rn(__fmul_rn(m.c1s, m1), __fsub_rn(pb, x));
  const float c = __fmul_rn(__fmul_rn(m.c2s, m2), __fsub_rn(g, x));
  float vn = __fadd_rn(__fadd_rn(a, b), c);
  vn = fminf(fmaxf(vn, vlo), vhi);
  x = fminf(fmaxf(__fadd_rn(x, vn), xlo), xhi);
  v = vn;
}

// Update one float4 (dims 4q..4q+3).  kB: bounds per dimension from the
// shared-memory table sB = [vlo | vhi | xlo | xhi] (nvec float4 each).
template <bool kB>
__device__ __forceinline__ void move4(const MoveParams& m, float4& x, float4& v, const float4& pb,
                                      const float4& g, const float4& r1, const float4& r2,
                                      const float4* sB, int nvec, int q) {
  if constexpr (kB) {
    const float4 vlo = sB[q], vhi = sB[nvec + q], xlo = sB[2 * nvec + q], xhi = sB[3 * nvec + q];
    move1b(m, x.x, v.x, pb.x, g.x, r1.x, r2.x, vlo.x, vhi.x, xlo.x, xhi.x);
    move1b(m, x.y, v.y, pb.y, g.y, r1.y, r2.y, vlo.y, vhi.y, xlo.y, xhi.y);
    move1b(m, x.z, v.z, pb.z, g.z, r1.z, r2.z, vlo.z, vhi.z, xlo.z, xhi.z);
    move1b(m, x.w, v.w, pb.w, g.w, r1.w, r2.w, vlo.w, vhi.w, xlo.w, xhi.w);
  } else {
    move1(m, x.x, v.x, pb.x, g.x, r1.x, r2.x);
    move1(m, x.y, v.y, pb.y, g.y, r1.y, r2.y);
    move1(m, x.z, v.z, pb.z, g.z, r1.z, r2.z);
    move1(m, x.w, v.w, pb.w, g.w, r1.w, r2.w);
  }
}

// Eq. 1 split at the gbest term, for work that overlaps the gbest exchange:
// the pre part (ab = w v + (c1 r1)(pb - x)) needs no gbest, the post part
// adds (c2 r2)(g - x), clamps and moves.  pre then post is move1 / move1b
// operation for operation (same roundings, same order).
__device__ __forceinline__ float move_pre1(const MoveParams& m, float x, float v, float pb, float m1) {
  return __fadd_rn(__fmul_rn(m.w, v), __fmul_rn(__fmul_rn(m.c1s, m1), __fsub_rn(pb, x)));
}
template <bool kB>
__device__ __forceinline__ void move_pre4(const MoveParams& m, const float4& x, const float4& v,
                                          const float4& pb, const float4& r1, float4& ab) {
  ab.x = move_pre1(m, x.x, v.x, pb.x, r1.x);
  ab.y = move_pre1(m, x.y, v.y, pb.y, r1.y);
  ab.z = move_pre1(m, x.z, v.z, pb.z, r1.z);
  ab.w = move_pre1(m, x.w, v.w, pb.w, r1.w);
}
__device__ __forceinline__ void move_post1(const MoveParams& m, float& x, float& v, float g, float m2,
                                           float ab, float vlo, float vhi, float xlo, float xhi) {
  const float c = __fmul_rn(__fmul_rn(m.c2s, m2), __fsub_rn(g, x));
  float vn = __fadd_rn(ab, c);
  vn = fminf(fmaxf(vn, vlo), vhi);
  x = fminf(fmaxf(__fadd_rn(x, vn), xlo), xhi);
  v = vn;
}
template <bool kB>
__device__ __forceinline__ void move_post4(const MoveParams& m, float4& x, float4& v, const float4& g,
                                           const float4& r2, const float4& ab, const float4* sB,
                                           int nvec, int q) {
  if constexpr (kB) {
    const float4 vlo = sB[q], vhi = sB[nvec + q], xlo = sB[2 * nvec + q], xhi = sB[3 * nvec + q];
    move_post1(m, x.x, v.x, g.x, r2.x, ab.x, vlo.x, vhi.x, xlo.x, xhi.x);
    move_post1(m, x.y, v.y, g.y, r2.y, ab.y, vlo.y, vhi.y, xlo.y, xhi.y);
    move_post1(m, x.z, v.z, g.z, r2.z, ab.z, vlo.z, vhi.z, xlo.z, xhi.z);
    move_post1(m, x.w, v.w, g.w, r2.w, ab.w, vlo.w, vhi.w, xlo.w, xhi.w);
  } else {
    move_post1(m, x.x, v.x, g.x, r2.x, ab.x, -m.vmax, m.vmax, m.lo, m.hi);
    move_post1(m, x.y, v.y, g.y, r2.y, ab.y, -m.vmax, m.vmax, m.lo, m.hi);
    move_post1(m, x.z, v.z, g.z, r2.z, ab.z, -m.vmax, m.vmax, m.lo, m.hi);
    move_post1(m, x.w, v.w, g.w, r2.w, ab.w, -m.vmax, m.vmax, m.lo, m.hi);
  }
}

// Row visiting order of the streaming kernels.  Rows are independent within an
// iteration and every cross-row result (candidate key, counters) is an
// order-free min / sum, so the order changes no bit.  Serpentine (a.serp):
// odd iterations walk the rows backwards, so an iteration starts on the rows
// the previous one wrote last -- still in L2 when the state is near its size.
struct RowOrder {
  long long n;
  bool rev;
  __device__ __forceinline__ long long operator()(long long i) const { return rev ? n - 1 - i : i; }
};
__device__ __forceinline__ RowOrder row_order(const SwarmArgs& a, uint32_t t) {
  return RowOrder{a.n_local, a.serp != 0 && (t & 1u) != 0};
}

// One float4 of a staged row with its random draws (A1-A4).  fl: lazy pbest
// row, PB == X bitwise (pbs is then not read).  x is finite there (every x the
// kernels store is clamped to finite bounds), so pb - x = +0 and
// (c1 r1)(pb - x) = copysign(0, c1) whatever r1 is: R1 is not drawn, and the
// result is move4's bit for bit -- a + (+-0) is still rounded as the oracle
// rounds it (-0 + +0 = +0).  Rows that improved the iteration before are lazy,
// so a converging swarm (C4: every row, every iteration) skips a quarter of the
// per-element instructions.
template <bool kB, class K>
__device__ __forceinline__ void move4_draw(const MoveParams& m, const K& key, uint32_t t, uint32_t gi,
                                           uint32_t q, int fl, float4& x, float4& v,
                                           const float4* pbs, const float4& g, const float4* sB,
                                           int nb, int qb) {
  if (fl) {
    const float4 r2 = raw24x4(key, kTagR2, t, gi, q);
    const float bz = copysignf(0.f, m.c1s);
    float4 ab;
    ab.x = __fadd_rn(__fmul_rn(m.w, v.x), bz);
    ab.y = __fadd_rn(__fmul_rn(m.w, v.y), bz);
    ab.z = __fadd_rn(__fmul_rn(m.w, v.z), bz);
    ab.w = __fadd_rn(__fmul_rn(m.w, v.w), bz);
    move_post4<kB>(m, x, v, g, r2, ab, sB, nb, qb);
  } else {
    const float4 pb = *pbs;
    const float4 r1 = raw24x4(key, kTagR1, t, gi, q);
    const float4 r2 = raw24x4(key, kTagR2, t, gi, q);
    move4<kB>(m, x, v, pb, g, r1, r2, sB, nb, qb);
  }
}

// move4_draw with the row-independent Philox rounds precomputed per thread
// slot (philox.cuh PhiloxSlot): the same draws bit for bit.
template <bool kB, class K>
__device__ __forceinline__ void move4_draw_slot(const MoveParams& m, const K& key, const PhiloxIter& it,
                                                const PhiloxSlot& s1, const PhiloxSlot& s2,
                                                uint32_t gi, int fl, float4& x, float4& v,
                                                const float4* pbs, const float4& g, const float4* sB,
                                                int nb, int qb) {
  uint32_t lo0r1, hi1r2, lo1r2;
  philox_row_shared(it, s2, gi, lo0r1, hi1r2, lo1r2);
  const float4 r2 = raw24x4(philox_slot_row(key, s2, lo0r1, hi1r2, lo1r2));
  if (fl) {
    const float bz = copysignf(0.f, m.c1s);
    float4 ab;
    ab.x = __fadd_rn(__fmul_rn(m.w, v.x), bz);
    ab.y = __fadd_rn(__fmul_rn(m.w, v.y), bz);
    ab.z = __fadd_rn(__fmul_rn(m.w, v.z), bz);
    ab.w = __fadd_rn(__fmul_rn(m.w, v.w), bz);
    move_post4<kB>(m, x, v, g, r2, ab, sB, nb, qb);
  } else {
    const float4 pb = *pbs;
    const float4 r1 = raw24x4(philox_slot_row(key, s1, lo0r1, hi1r2, lo1r2));
    move4<kB>(m, x, v, pb, g, r1, r2, sB, nb, qb);
  }
}

// --- CTA reduction of the functor accumulators -----------------------------
template <class Obj>
__device__ __forceinline__ void warp_combine(float* a) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    float b[Obj::kAcc];
#pragma unroll
    for (int k = 0; k < Obj::kAcc; ++k) b[k] = __shfl_xor_sync(kFull, a[k], off);
    Obj::combine(a, b);
  }
}

// Shared scratch of the row pipeline.
template <class Obj>
struct RowSmem {
  float red[32 * Obj::kAcc];
  float f;
  int improved;
  int last;
  unsigned long long gbar;      // gbest staging barrier
  unsigned long long acc, cur;  // epilogue scratch (adjacent: sh[0], sh[1])
  unsigned long long inc;       // exchange: merged incumbent of the previous iteration
  int src;                      // exchange: rank whose record won (-1: none)
};

// Reduce a[] over the nthr compute threads (fixed order: lanes by
// xor-butterfly, then warps in index order), finalize in thread 0 and decide
// the pbest update against pf_old (only thread 0's pf_old is read).
template <class Obj>
__device__ __forceinline__ float cta_fitness(float* a, RowSmem<Obj>& sm, int d, float pf_old,
                                             bool& improved, int tid, int nthr) {
  warp_combine<Obj>(a);
  const int warp = tid >> 5, lane = tid & 31;
  if (lane == 0) {
#pragma unroll
    for (int k = 0; k < Obj::kAcc; ++k) sm.red[warp * Obj::kAcc + k] = a[k];
  }
  team_sync(nthr);
  if (warp == 0) {
    float c[Obj::kAcc];
    Obj::init(c);
    if (lane < (nthr >> 5)) {
#pragma unroll
      for (int k = 0; k < Obj::kAcc; ++k) c[k] = sm.red[lane * Obj::kAcc + k];
    }
    warp_combine<Obj>(c);
    if (lane == 0) {
      const float f = Obj::finalize(c, d);
      sm.f = f;
      sm.improved = (f < pf_old) ? 1 : 0;  // strict; NaN never improves
    }
  }
  team_sync(nthr);
  improved = sm.improved != 0;
  return sm.f;
}

// Map one float4 of new positions (dims j..j+3; nx = x_{j+4} for neighbours).
template <class Obj, class = void>
struct HasRowTable : std::false_type {};
template <class Obj>
struct HasRowTable<Obj, std::enable_if_t<Obj::kRowTable>> : std::true_type {};

template <class Obj, class = void>
struct HasMap4 {
  static constexpr bool value = false;
};
template <class Obj>
struct HasMap4<Obj, decltype(Obj::map4(nullptr, float4{}, 0.f, 0, 0))> {
  static constexpr bool value = true;
};
template <class Obj>
__device__ __forceinline__ void map4(float* acc, const float4& x, float nx, int j, int d) {
  if (j + 3 < d) {
    if constexpr (HasMap4<Obj>::value) {
      Obj::map4(acc, x, nx, j, d);
    } else {
      Obj::map(acc, x.x, x.y, j, d);
      Obj::map(acc, x.y, x.z, j + 1, d);
      Obj::map(acc, x.z, x.w, j + 2, d);
      Obj::map(acc, x.w, nx, j + 3, d);
    }
  } else {  // ragged tail of the row
    if (j < d) Obj::map(acc, x.x, x.y, j, d);
    if (j + 1 < d) Obj::map(acc, x.y, x.z, j + 1, d);
    if (j + 2 < d) Obj::map(acc, x.z, x.w, j + 2, d);
  }
}

// Map the VPT float4 of new positions into the accumulators.  For functors
// that need x_{j+1} the first element of every float4 is published in sFirst.
template <class Obj, int VPT>
__device__ __forceinline__ void map_row(float* acc, const float4 (&x)[VPT], float* sFirst,
                                        int nvec, int d, int tid, int nthr) {
  if constexpr (Obj::kNeighbor) {
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = tid + s * nthr;
      if (q < nvec) sFirst[q] = x[s].x;
    }
    team_sync(nthr);
  }
#pragma unroll
  for (int s = 0; s < VPT; ++s) {
    const int q = tid + s * nthr;
    if (q < nvec) {
      float nx = 0.f;
      if constexpr (Obj::kNeighbor) nx = (q + 1 < nvec) ? sFirst[q + 1] : 0.f;
      map4<Obj>(acc, x[s], nx, 4 * q, d);
    }
  }
}


// A2-A6 for one row: update, store x' / v', evaluate, pbest compare-and-copy.
// src(s, q, x, v, pb) supplies the operands of float4 q (slot s) — from
// registers (k_step_reg) or from the shared-memory stage (k_step_tma);
// release() runs once every operand has been read.  x' stays in registers
// (xn) until the pbest decision.  Returns f; `improved` is CTA-uniform.
template <class Obj, int VPT, bool kB, class Src, class Release, class K>
__device__ __forceinline__ float process_row(const SwarmArgs& a, const MoveParams& mp,
                                             const K& key, uint32_t t, uint32_t gi, long long r,
                                             Src&& src, Release&& release, const float4* sG,
                                             const float4* sB,
                                             float* sFirst, RowSmem<Obj>& sm, int tid, int nthr,
                                             float pf_old, bool& improved) {
  const int nvec = a.nvec, d = a.d;
  float4* Xr = reinterpret_cast<float4*>(a.X) + r * nvec;
  float4* Vr = reinterpret_cast<float4*>(a.V) + r * nvec;
  float4* Pr = reinterpret_cast<float4*>(a.PB) + r * nvec;
  float4 xn[VPT];
#pragma unroll
  for (int s = 0; s < VPT; ++s) {
    const int q = tid + s * nthr;
    if (q < nvec) {
      float4 x, v, pb;
      src(s, q, x, v, pb);
      const float4 g = sG[q];
      const float4 r1 = raw24x4(key, kTagR1, t, gi, (uint32_t)q);
      const float4 r2 = raw24x4(key, kTagR2, t, gi, (uint32_t)q);
      move4<kB>(mp, x, v, pb, g, r1, r2, sB, nvec, q);
      if ((d & 3) && q == nvec - 1) {  // keep the row padding at zero
        const int j = 4 * q;
        if (j + 1 >= d) x.y = v.y = 0.f;
        if (j + 2 >= d) x.z = v.z = 0.f;
        if (j + 3 >= d) x.w = v.w = 0.f;
      }
      st_stream(Xr + q, x);
      st_stream(Vr + q, v);
      xn[s] = x;
    }
  }
  release();
  float acc[Obj::kAcc];
  Obj::init(acc);
  map_row<Obj, VPT>(acc, xn, sFirst, nvec, d, tid, nthr);
  const float f = cta_fitness<Obj>(acc, sm, d, pf_old, improved, tid, nthr);
  if (improved) {
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = tid + s * nthr;
      if (q < nvec) st_stream(Pr + q, xn[s]);
    }
  }
  return f;
}

// --- gbest exchange (world > 1, or forced): records of iteration t live in
// recv[t & 1][rank] = {u64 key, u64 tag, pitch floats}.  The step kernel of
// iteration t + 1 merges them in its prologue (the incumbent for its strict
// filter and the G it stages); its last CTA commits that merge to key_cur / G
// and publishes the new local candidate.
// Records are kept for 4 iterations (slot t & 3): the asynchronous mode reads
// iteration t - 2 while a peer that is one iteration ahead writes t + 1.
__device__ __forceinline__ const unsigned char* records(const SwarmArgs& a, uint32_t t) {
  return a.recv + (size_t)(t & 3u) * a.world * record_bytes(a.nvec * 4);
}
// The iteration whose records the step kernel of iteration t merges:
// synchronous t - 1; asynchronous (NEXT-4, "updated in an asynchronous
// manner") t - 2, so a rank never waits for the iteration its peers are in --
// but never before t_base, the iteration of the last synchronous re-selection
// (create: 0, set_state: its t), the oldest records of the current epoch.
__device__ __forceinline__ uint32_t merge_iter(const SwarmArgs& a, uint32_t t) {
  return a.async_gbest ? (t >= a.t_base + 2u ? t - 2u : a.t_base) : t - 1u;
}
// --- NVLink peer exchange (p2p): every rank stores its record of iteration
// t straight into recv[t & 1][rank] of every peer (CUDA-IPC-mapped), then the
// record's tag with release semantics at system scope; readers acquire the
// tags.  No collective call and no host involvement per iteration.
__device__ __forceinline__ unsigned long long ld_acquire_sys_u64(const void* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys_u64(void* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Wait until every rank's record of iteration t has landed (one thread).  A
// peer that never delivers (a crashed rank) traps after 60 s instead of
// hanging the GPU.
__device__ __forceinline__ void wait_records(const SwarmArgs& a, uint32_t t) {
  const size_t rec = record_bytes(a.nvec * 4);
  const unsigned char* base = records(a, t);
  const unsigned long long t0 = globaltimer_ns();
  for (int r = 0; r < a.world; ++r) {
    const void* tag = base + (size_t)r * rec + 8;
    const unsigned long long want = ((unsigned long long)a.epoch << 32) | t;
    while (ld_acquire_sys_u64(tag) != want) {
      __nanosleep(64);
      if (globaltimer_ns() - t0 > a.peer_timeout_ns) __trap();
    }
  }
  fence_proxy_async_global();  // the records are then read by bulk copies too
}

// Minimum of the incumbent and the records of iteration prev_t; *src = the
// winning rank, or -1 when nothing beat the incumbent.  One thread.
__device__ __forceinline__ unsigned long long exchange_merge(const SwarmArgs& a, uint32_t prev_t,
                                                             int* src) {
  if (a.p2p) wait_records(a, prev_t);
  const size_t rec = record_bytes(a.nvec * 4);
  const unsigned char* base = records(a, prev_t);
  const unsigned long long cur = *(volatile unsigned long long*)&a.ctl->key_cur;
  unsigned long long best = cur;
  int s = -1;
  for (int r = 0; r < a.xrecs; ++r) {
    const unsigned long long k = *reinterpret_cast<const unsigned long long*>(base + (size_t)r * rec);
    // strictly better fitness than the incumbent (Alg. 1 line 10), then the
    // lowest key: in the synchronous mode every record already satisfies it
    if ((k >> 32) < (cur >> 32) && k < best) {
      best = k;
      s = r;
    }
  }
  *src = s;
  return best;
}
// The same merge by a whole warp (the producer warp of the TMA and cluster
// kernels): lane r waits for and reads rank r's record, so the world's tags
// and keys cost one round trip instead of one each; a shuffle takes the
// minimum (keys are unique: global particle indices).  __syncwarp orders
// every lane's acquire before lane 0's bulk copy of the winning row.
__device__ __forceinline__ unsigned long long exchange_merge_warp(const SwarmArgs& a, uint32_t prev_t,
                                                                  int lane, int* src) {
  const size_t rec = record_bytes(a.nvec * 4);
  const unsigned char* base = records(a, prev_t);
  const unsigned long long want = ((unsigned long long)a.epoch << 32) | prev_t;
  const unsigned long long cur = *(volatile unsigned long long*)&a.ctl->key_cur;
  const unsigned long long t0 = globaltimer_ns();
  unsigned long long best = cur;
  int s = -1;
  for (int r = lane; r < a.xrecs; r += 32) {
    if (a.p2p) {
      while (ld_acquire_sys_u64(base + (size_t)r * rec + 8) != want) {
        __nanosleep(64);
        if (globaltimer_ns() - t0 > a.peer_timeout_ns) __trap();
      }
    }
    const unsigned long long k = *reinterpret_cast<const volatile unsigned long long*>(base + (size_t)r * rec);
    if ((k >> 32) < (cur >> 32) && k < best) {  // strictly better fitness, then the lowest key
      best = k;
      s = r;
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    const unsigned long long ob = __shfl_xor_sync(kFull, best, off);
    const int os = __shfl_xor_sync(kFull, s, off);
    if (ob < best) {
      best = ob;
      s = os;
    }
  }
  __syncwarp();
  if (a.p2p) fence_proxy_async_global();  // the records are then read by bulk copies too
  *src = s;
  return best;
}
__device__ __forceinline__ const float* merged_gbest_row(const SwarmArgs& a, uint32_t prev_t, int src) {
  return src < 0 ? a.G
                 : reinterpret_cast<const float*>(records(a, prev_t) +
                                                  (size_t)src * record_bytes(a.nvec * 4) + 16);
}

// Last-CTA epilogue of iteration t, run by `nthr` threads (tid 0 leads;
// `sync` orders them; `sh` is 2 words of shared scratch).
//   single GPU: copy PB[gi] into G and advance the incumbent key.
//   exchange:   commit the prologue's merge (inc from rank `src`) to key_cur /
//               G, then write the local candidate record (strictly below inc)
//               for the all-gather, tagged with t; reset the accumulator.
// `rows` holds the winning candidate's position: X for the step and init
// kernels (a candidate improved, so its x' is its pbest), PB for rebest.
template <class SyncF>
__device__ __forceinline__ void epilogue_core(const SwarmArgs& a, uint32_t t, unsigned long long inc,
                                              int src, unsigned long long* sh, int tid, int nthr,
                                              SyncF sync, const float* rows) {
  if (tid == 0) {
    __threadfence();
    sh[0] = *(volatile unsigned long long*)&a.ctl->key_acc;
    sh[1] = a.ctl->key_cur;
  }
  sync();
  const unsigned long long acc = sh[0], cur = sh[1];
  float4* G4 = reinterpret_cast<float4*>(a.G);
  if (!a.exchange) {
    const bool have = acc < cur;
    if (have) {
      const float4* pb = reinterpret_cast<const float4*>(rows) +
                         ((long long)(uint32_t)acc - a.row_begin) * a.nvec;
      for (int q = tid; q < a.nvec; q += nthr) G4[q] = __ldcg(pb + q);
    }
    if (tid == 0) {
      if (have) a.ctl->key_cur = acc;
      a.ctl->t = t;
      a.ctl->done = 0;
    }
    return;
  }
  const bool merged = src >= 0 && inc < cur;
  const bool have = acc != ~0ull;
  // asynchronous: this rank's candidate becomes its incumbent at once (it is
  // strictly below the merged incumbent); synchronous: every rank adopts it
  // through the next merge
  const bool local = a.async_gbest && have;
  if (merged && !local) {
    const float4* w = reinterpret_cast<const float4*>(merged_gbest_row(a, merge_iter(a, t), src));
    for (int q = tid; q < a.nvec; q += nthr) G4[q] = __ldcg(w + q);
  }
  if (local) {
    const float4* w = reinterpret_cast<const float4*>(rows) +
                      ((long long)(uint32_t)acc - a.row_begin) * a.nvec;
    for (int q = tid; q < a.nvec; q += nthr) G4[q] = __ldcg(w + q);
  }
  const float4* pb = have ? reinterpret_cast<const float4*>(rows) +
                                ((long long)(uint32_t)acc - a.row_begin) * a.nvec
                          : nullptr;
  const unsigned long long key = have ? acc : ~0ull;
  if (!a.p2p) {  // NCCL: the host all-gathers `send`
    if (have) {
      float4* row = reinterpret_cast<float4*>(a.send + 16);
      for (int q = tid; q < a.nvec; q += nthr) row[q] = __ldcg(pb + q);
    }
    if (tid == 0) {
      unsigned long long* hdr = reinterpret_cast<unsigned long long*>(a.send);
      hdr[0] = key;
      // the same (epoch, iteration) tag as the NVLink records, so a handle that
      // switches to p2p after set_state finds its last all-gathered records
      hdr[1] = ((unsigned long long)a.epoch << 32) | t;
    }
  } else {  // NVLink: store the record into recv[t & 1][rank] of every rank
    // the row is read once and stored to every rank; thread r releases rank r's tag
    const size_t rec = record_bytes(a.nvec * 4);
    const size_t off = (size_t)(t & 3u) * a.world * rec + (size_t)a.rank * rec;
    if (have) {
      for (int q = tid; q < a.nvec; q += nthr) {
        const float4 v = __ldcg(pb + q);
        for (int r = 0; r < a.world; ++r) reinterpret_cast<float4*>(a.peers[r] + off + 16)[q] = v;
      }
    }
    for (int r = tid; r < a.world; r += nthr) reinterpret_cast<unsigned long long*>(a.peers[r] + off)[0] = key;
    // One system-scope fence per tag: the release store's own.  `sync` orders
    // every thread's record stores before it (barrier), and the release is
    // cumulative over them.  (A __threadfence_system() in every thread before
    // the barrier doubled the fences: +3.4 us per iteration.)
    sync();
    // (Measured, round 2: this system-scope release costs 1.7 us per iteration on
    // the one-GPU proxy -- NS_R8 with the exchange forced 82.9 us, 81.2 us with a
    // relaxed store in its place, 79.0 us without the exchange.)
    for (int r = tid; r < a.world; r += nthr)
      st_release_sys_u64(a.peers[r] + off + 8, ((unsigned long long)a.epoch << 32) | t);
  }
  if (tid == 0) {
    if (local)
      a.ctl->key_cur = acc;
    else if (merged)
      a.ctl->key_cur = inc;
    a.ctl->key_acc = ~0ull;
    a.ctl->t = t;
    a.ctl->done = 0;
  }
}

template <class Obj>
__device__ __forceinline__ void gbest_epilogue(const SwarmArgs& a, RowSmem<Obj>& sm, uint32_t t,
                                               int tid, int nthr, unsigned long long inc = ~0ull,
                                               int src = -1, const float* rows = nullptr) {
  epilogue_core(a, t, inc, src, &sm.acc, tid, nthr, [&] { team_sync(nthr); }, rows ? rows : a.X);
}

// The same epilogue run by one warp (the finaliser warp of the TMA kernels).
__device__ __forceinline__ void warp_gbest_epilogue(const SwarmArgs& a, uint32_t t, int lane,
                                                    unsigned long long inc = ~0ull, int src = -1) {
  __shared__ unsigned long long sh[2];
  epilogue_core(a, t, inc, src, sh, lane, 32, [] { __syncwarp(); }, a.X);
}

// Publish this CTA's candidate and improvement count; true in the last CTA
// to finish (which then runs gbest_epilogue).
template <class Obj>
__device__ __forceinline__ bool cta_finish(const SwarmArgs& a, RowSmem<Obj>& sm,
                                           unsigned long long best, unsigned nimp, int tid,
                                           int nthr) {
  team_sync(nthr);  // every PB / X / V store of this CTA is issued
  if (tid == 0) {
    if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
    if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
    __threadfence();
    const unsigned ticket = atomicAdd(&a.ctl->done, 1u);
    sm.last = (ticket == gridDim.x - 1) ? 1 : 0;
  }
  team_sync(nthr);
  return sm.last != 0;
}

__device__ __forceinline__ void row_bookkeeping(const SwarmArgs& a, long long r, uint32_t gi,
                                                float f, bool improved, uint32_t inc_ord,
                                                unsigned long long& best, unsigned& nimp) {
  if (improved) {
    a.pf[r] = f;
    ++nimp;
  }
  if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
    const unsigned long long k = pack_key(f, gi);
    best = k < best ? k : best;
  }
}

// ------------------------------------------------- step kernel: registers
template <class Obj, int VPT, bool kB>
__global__ void __launch_bounds__(kMaxThreads, (VPT >= 8) ? 1 : 2)
    k_step_reg(const __grid_constant__ SwarmArgs a, int /*stages: unused, same signature as k_step_tma*/) {
  extern __shared__ __align__(128) unsigned char dsmem[];
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float4* sB = sG + a.nvec;  // kB: [vlo | vhi | xlo | xhi]
  float* sFirst = reinterpret_cast<float*>(sB + (kB ? 4 * a.nvec : 0));
  __shared__ RowSmem<Obj> sm;
  const int tid = threadIdx.x, nthr = blockDim.x;
  pdl_wait_and_release();
  const uint32_t t = a.ctl->t + 1u;
  if (tid == 0) {
    const unsigned row_bytes = (unsigned)a.nvec * 16u;
    const float* gsrc = a.G;
    sm.src = -1;
    sm.inc = a.ctl->key_cur;
    if (a.exchange) {  // merge the previous iteration's records (the all-gather)
      sm.inc = exchange_merge(a, merge_iter(a, t), &sm.src);
      gsrc = merged_gbest_row(a, merge_iter(a, t), sm.src);
    }
    mbar_init(&sm.gbar, 1);
    mbar_fence_init();
    mbar_expect_tx(&sm.gbar, row_bytes * (kB ? 5u : 1u));
    bulk_g2s(sG, gsrc, row_bytes, &sm.gbar);
    if (kB) bulk_g2s(sB, a.bounds, 4u * row_bytes, &sm.gbar);
  }
  __syncthreads();
  const uint32_t inc_ord = (uint32_t)(sm.inc >> 32);
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  const int nvec = a.nvec;
  // Rows are loaded one row ahead (VPT <= 2: the registers are there): the L2 /
  // DRAM latency of row r + grid overlaps row r's arithmetic and reduction, and
  // the first row's loads overlap the gbest staging.  The paper's default
  // experiment (Sphere 5000 x 200, L2-resident): 9.1 -> 8.7 us per iteration.
  constexpr bool kAhead = VPT <= 2;
  float4 xn[VPT], vn[VPT], pbn[VPT];
  float pfn = 0.f;
  auto load_row = [&](long long r, float4 (&xo)[VPT], float4 (&vo)[VPT], float4 (&po)[VPT], float& pfo) {
    const float4* Xr = reinterpret_cast<const float4*>(a.X) + r * nvec;
    const float4* Vr = reinterpret_cast<const float4*>(a.V) + r * nvec;
    const float4* Pr = reinterpret_cast<const float4*>(a.PB) + r * nvec;
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = tid + s * nthr;
      if (q < nvec) {
        xo[s] = ld_stream(Xr + q);
        vo[s] = ld_stream(Vr + q);
        po[s] = ld_stream(Pr + q);
      }
    }
    pfo = (tid == 0) ? a.pf[r] : 0.f;
  };
  if (kAhead && blockIdx.x < a.n_local) load_row(blockIdx.x, xn, vn, pbn, pfn);
  mbar_wait(&sm.gbar, 0);

  unsigned long long best = ~0ull;
  unsigned nimp = 0;
  for (long long r = blockIdx.x; r < a.n_local; r += gridDim.x) {
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    float4 x[VPT], v[VPT], pb[VPT];
    float pf_old;
    if constexpr (kAhead) {
#pragma unroll
      for (int s = 0; s < VPT; ++s) {
        x[s] = xn[s];
        v[s] = vn[s];
        pb[s] = pbn[s];
      }
      pf_old = pfn;
      if (r + gridDim.x < a.n_local) load_row(r + gridDim.x, xn, vn, pbn, pfn);
    } else {
      load_row(r, x, v, pb, pf_old);
    }
    bool improved;
    const float f = process_row<Obj, VPT, kB>(
        a, mp, key, t, gi, r,
        [&](int s, int, float4& xo, float4& vo, float4& po) {
          xo = x[s];
          vo = v[s];
          po = pb[s];
        },
        [] {}, sG, sB, sFirst, sm, tid, nthr, pf_old, improved);
    if (tid == 0) row_bookkeeping(a, r, gi, f, improved, inc_ord, best, nimp);
  }
  if (tid == 0) {  // traffic counters: every pbest row read, improved ones written
    const long long rows = (a.n_local - blockIdx.x + gridDim.x - 1) / gridDim.x;
    if (rows > 0) atomicAdd(&a.ctl->pb_loads, (unsigned long long)rows);
    if (nimp) atomicAdd(&a.ctl->pb_stores, (unsigned long long)nimp);
  }
  if (cta_finish<Obj>(a, sm, best, nimp, tid, nthr))
    gbest_epilogue<Obj>(a, sm, t, tid, nthr, sm.inc, sm.src);
}

// ------------------------------------------------- step kernel: TMA pipeline
// Warp-specialised; every HBM byte of the row stream moves through the TMA
// engine (bulk async copies), the compute warps touch only shared memory.
//   warps 0..W-1  compute: x, v, pb, g from the stage (LDS.128) -> Philox ->
//                 Eq. 1/5/2 -> x', v' written back into the stage (STS.128)
//                 -> objective map -> warp partial -> arrive(done[s])
//   warp  W       producer: G once, then per row cp.async.bulk x, v, pb rows
//                 global -> stage s, completion on full[s] (complete_tx)
//   warp  W+1     finaliser: per row, combine the W warp partials (fixed
//                 order), f, the pbest decision, then bulk-store the stage's
//                 x' -> X, v' -> V (and x' -> PB if improved), the gbest
//                 candidate, and release the stage to the producer once the
//                 bulk stores have read it (wait_group.read).
// Barriers per stage: full (1 arrival + tx bytes), done (W arrivals), empty (1).
// Shared memory: [G: nvec float4][stages x {x, v, pb}: nvec float4 each].
// kMaxT: compute threads the instantiation is built for -- 256 (two CTAs per
// SM) or 512 (the wide variant: one CTA of 16 compute warps per SM, for rows
// of 513-2048 float4 whose stages do not fit twice).
template <class Obj, int VPT, bool kB, int kMaxT = kMaxThreads>
__global__ void __launch_bounds__(kMaxT + 64, kMaxT > kMaxThreads ? 1 : 2)
    k_step_tma(const __grid_constant__ SwarmArgs a, int stages) {
  extern __shared__ __align__(128) unsigned char dsmem[];
  const int nvec = a.nvec, d = a.d;
  const int nthr = (int)blockDim.x - 64;  // compute threads
  const int nwarps = nthr >> 5;
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float4* sB = sG + nvec;  // kB: [vlo | vhi | xlo | xhi]
  float4* ring = sB + (kB ? 4 * nvec : 0);
  __shared__ float red[kMaxStages][(kMaxT / 32) * 2];
  __shared__ unsigned long long full[kMaxStages], empty[kMaxStages], done[kMaxStages], gbar;
  __shared__ unsigned long long s_inc;  // incumbent of this iteration (after the exchange merge)
  __shared__ int s_src;
  __shared__ int sflag[kMaxStages];     // lazy pbest: the stage's row had PB == X (pb not loaded)
  __shared__ long long srow[kMaxStages];  // the stage's row (local index), -1: no more rows
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    mbar_init(&gbar, 1);
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&done[s], (unsigned)nwarps);
      mbar_init(&empty[s], 1);
    }
    mbar_fence_init();
  }
  __syncthreads();
  pdl_wait_and_release();
  const uint32_t t = a.ctl->t + 1u;
  const unsigned row_bytes = (unsigned)nvec * 16u;

  if (warp == nwarps) {  // ---------------- producer
    int xsrc = -1;
    unsigned long long xinc = 0;
    if (a.exchange) xinc = exchange_merge_warp(a, merge_iter(a, t), lane, &xsrc);  // the all-gather's merge
    if (lane == 0) {
      const float* gsrc = a.G;
      s_src = -1;
      s_inc = a.ctl->key_cur;
      if (a.exchange) {
        s_inc = xinc;
        s_src = xsrc;
        gsrc = merged_gbest_row(a, merge_iter(a, t), xsrc);
      }
      mbar_expect_tx(&gbar, row_bytes * (kB ? 5u : 1u));  // releases s_inc / s_src too
      bulk_g2s(sG, gsrc, row_bytes, &gbar);
      if (kB) bulk_g2s(sB, a.bounds, 4u * row_bytes, &gbar);
      int s = 0;
      unsigned ph = 0;
      int k = 0;
      // lazy pbest: rows whose PB equals X skip the pb load (flag prefetched one row ahead)
      const RowOrder ro = row_order(a, t);
      const long long n = a.n_local;
      // Row schedule.  Round robin (row i to CTA i mod grid), or dynamic: a
      // CTA's first row is its blockIdx, every further one is claimed from
      // ctl->row_claim, so CTAs that run faster (SM placement, the co-resident
      // CTA's lazy-row share) take more rows and the grid ends together.  A
      // claim is issued two rows ahead (its value is needed one row ahead, for
      // the lazy flag) and only while the previous claim was a row, so every
      // claim's value is consumed before the sentinel below: the last CTA's
      // reset of the counter then follows every claim of the iteration.  Which
      // CTA computes a row changes no bit (rows are independent; the candidate
      // key and the counters are order-free min / sums).
      unsigned long long* claim_ctr = &a.ctl->row_claim;
      const bool dyn = (a.dyn_rows & 1) != 0;
      long long i = blockIdx.x;
      long long i_next =
          i >= n ? n : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + gridDim.x : i + gridDim.x);
      int fl_next = (a.lazy_pb && i < n) ? a.pbx[ro(i)] : 0;
      // L2 prefetch of the row l2pf rounds of the grid beyond the load front:
      // DRAM requests in flight beyond the ring.  Only lazy rows by default --
      // their stage loads 2 of its 3 slots, so the ring alone keeps a third
      // fewer bytes in flight (C4: 547 -> 529 us); prefetching eager rows as
      // well slows the ring-saturated case (NS 638 -> 671 us).  Flag read one
      // row earlier.  (Dynamic rows: the prefetched row is claimed by whichever
      // CTA reaches it; L2 is shared.)
      const long long pd = (long long)a.l2pf * gridDim.x;
      int pfl_next = (pd && i + pd < n) ? a.pbx[ro(i + pd)] : 0;
      for (; i < n; ++k) {
        const long long r = ro(i);
        const int fl = fl_next;
        const long long i_nn = i_next >= n ? n
                               : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + gridDim.x
                                      : i_next + gridDim.x);
        if (a.lazy_pb && i_next < n) fl_next = a.pbx[ro(i_next)];
        if (pd && i + pd < n) {
          const int pfl = pfl_next;
          if (i_next + pd < n) pfl_next = a.pbx[ro(i_next + pd)];
          const size_t po = (size_t)ro(i + pd) * 4 * nvec;
          if (pfl || a.l2pf_all) {
            bulk_prefetch_l2(a.X + po, row_bytes);
            bulk_prefetch_l2(a.V + po, row_bytes);
            if (!pfl) bulk_prefetch_l2(a.PB + po, row_bytes);
          }
        }
        i = i_next;
        i_next = i_nn;
        if (k >= stages) mbar_wait(&empty[s], ph ^ 1u);
        float4* st = ring + (size_t)s * 3 * nvec;
        PSO_DCHECK(r >= 0 && r < n && s < stages && stages <= kMaxStages);
        PSO_DCHECK((size_t)((const unsigned char*)(st + 3 * nvec) - dsmem) <= dyn_smem_bytes());
        sflag[s] = fl;
        srow[s] = r;
        mbar_expect_tx(&full[s], (fl ? 2u : 3u) * row_bytes);  // releases sflag[s], srow[s] too
        bulk_g2s(st, a.X + (size_t)r * 4 * nvec, row_bytes, &full[s]);
        bulk_g2s(st + nvec, a.V + (size_t)r * 4 * nvec, row_bytes, &full[s]);
        if (!fl) bulk_g2s(st + 2 * nvec, a.PB + (size_t)r * 4 * nvec, row_bytes, &full[s]);
        if (++s == stages) {
          s = 0;
          ph ^= 1u;
        }
      }
      // sentinel: the compute warps and the finaliser stop at a stage without a row
      if (k >= stages) mbar_wait(&empty[s], ph ^ 1u);
      srow[s] = -1;
      mbar_arrive(&full[s]);
    }
    return;
  }

  if (warp == nwarps + 1) {  // ---------------- finaliser
    __shared__ int s_last;
    if (lane == 0) {
      mbar_wait(&gbar, 0);
      const uint32_t inc_ord = (uint32_t)(s_inc >> 32);
      unsigned long long best = ~0ull;
      unsigned nimp = 0, n_pbl = 0, n_pbs = 0;
      int s = 0, prev = -1;
      unsigned ph = 0;
      for (;;) {
        mbar_wait(&full[s], ph);
        const long long r = srow[s];
        if (r < 0) break;
        const float pf_old = a.pf[r];
        const uint32_t gi = (uint32_t)(a.row_begin + r);
        mbar_wait(&done[s], ph);
        float c[Obj::kAcc];
        Obj::init(c);
        for (int w = 0; w < nwarps; ++w) {
          float b[Obj::kAcc];
#pragma unroll
          for (int j = 0; j < Obj::kAcc; ++j) b[j] = red[s][w * Obj::kAcc + j];
          Obj::combine(c, b);
        }
        const float f = Obj::finalize(c, d);
        const float4* st = ring + (size_t)s * 3 * nvec;
        const size_t off = (size_t)r * 4 * nvec;
        const int fl = sflag[s];
        const float4* xnew = fl ? st + 2 * nvec : st;  // where the compute warps put x'
        const bool improved = f < pf_old;  // Alg. 1 line 7: strict; NaN never improves
        bulk_s2g(a.X + off, xnew, row_bytes);
        bulk_s2g(a.V + off, st + nvec, row_bytes);
        n_pbl += fl ? 0u : 1u;
        if (!a.lazy_pb) {
          if (improved) {
            bulk_s2g(a.PB + off, st, row_bytes);
            ++n_pbs;
          }
        } else {  // PB == X after an improvement: defer the copy until the row stops improving
          if (fl && !improved) {
            bulk_s2g(a.PB + off, st, row_bytes);  // st holds the old x
            ++n_pbs;
          }
          if ((int)improved != fl) a.pbx[r] = improved ? 1 : 0;
        }
        if (improved) {
          a.pf[r] = f;
          ++nimp;
        }
        bulk_commit();
        if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
          const unsigned long long key = pack_key(f, gi);
          best = key < best ? key : best;
        }
        // the previous row's stores have read their stage.  (Waiting for this
        // row's own stores instead releases stages a row earlier but blocks
        // the finaliser behind HBM writes: -1.7 % on C4, +7.7 % on NS.)
        if (prev >= 0) {
          bulk_wait_read<1>();
          mbar_arrive(&empty[prev]);
        }
        prev = s;
        if (++s == stages) {
          s = 0;
          ph ^= 1u;
        }
      }
      bulk_wait_all();  // every X / V / PB row written
      fence_proxy_async_global();
      if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
      if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
      if (n_pbl) atomicAdd(&a.ctl->pb_loads, (unsigned long long)n_pbl);
      if (n_pbs) atomicAdd(&a.ctl->pb_stores, (unsigned long long)n_pbs);
      __threadfence();
      s_last = (atomicAdd(&a.ctl->done, 1u) == gridDim.x - 1) ? 1 : 0;
      if (s_last) a.ctl->row_claim = 0;  // every CTA's claims are done (see the producer)
    }
    __syncwarp();
    if (s_last) warp_gbest_epilogue(a, t, lane, s_inc, s_src);
    return;
  }

  // ---------------- compute warps
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  // row-invariant functor factors of this thread's float4 slots (VPT <= 2: registers)
  constexpr bool kTab = HasRowTable<Obj>::value && !Obj::kNeighbor && VPT <= 2;
  float4 rtab[VPT];
  if constexpr (kTab) {
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int q = tid + j * nthr;
      rtab[j] = q < nvec ? Obj::table4(4 * q) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
  // row-invariant Philox rounds of this thread's slots (VPT <= 2: registers)
  // Wide (512-thread, 1 CTA/SM) instantiation: C5 12.62 -> 12.36 ms; 256-thread one:
  // see PSO_SLOT_PHILOX_NARROW (scalar bounds; not for neighbour functors: Rosenbrock
  // +11 registers)
  constexpr bool kSlotRng = PSO_SLOT_PHILOX && VPT <= 2 && !Obj::kNeighbor &&
                            (kMaxT > kMaxThreads || (PSO_SLOT_PHILOX_NARROW && !kB));
  const PhiloxIter pit = philox_iter(key, t);
  PhiloxSlot ps1[VPT], ps2[VPT];
  if constexpr (kSlotRng) {
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const uint32_t q = (uint32_t)(tid + j * nthr);
      ps1[j] = philox_slot(key, pit, q, kTagR1);
      ps2[j] = philox_slot(key, pit, q, kTagR2);
    }
  }
  mbar_wait(&gbar, 0);
  int s = 0;
  unsigned ph = 0;
  for (;;) {
    float4* st = ring + (size_t)s * 3 * nvec;
    mbar_wait(&full[s], ph);
    const long long r = srow[s];
    if (r < 0) break;
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    // lazy pbest row (PB == X): pb is the loaded x, and x' goes to the pb slot
    // so the old x stays available for a deferred PB store
    const int fl = sflag[s];
    float4* xdst = fl ? st + 2 * nvec : st;
    float acc[Obj::kAcc];
    Obj::init(acc);
    // VPT <= 2: fully unrolled for ILP; larger VPT: pairs, to bound registers.
#pragma unroll(VPT <= 2 ? VPT : 2)
    for (int j = 0; j < VPT; ++j) {
      const int q = tid + j * nthr;
      if (q < nvec) {
        float4 x = st[q], v = st[nvec + q];
        const float4 g = sG[q];
        if constexpr (kSlotRng)
          move4_draw_slot<kB>(mp, key, pit, ps1[j], ps2[j], gi, fl, x, v, st + 2 * nvec + q, g, sB, nvec, q);
        else
          move4_draw<kB>(mp, key, t, gi, (uint32_t)q, fl, x, v, st + 2 * nvec + q, g, sB, nvec, q);
        if ((d & 3) && q == nvec - 1) {  // keep the row padding at zero
          const int jj = 4 * q;
          if (jj + 1 >= d) x.y = v.y = 0.f;
          if (jj + 2 >= d) x.z = v.z = 0.f;
          if (jj + 3 >= d) x.w = v.w = 0.f;
        }
        xdst[q] = x;
        st[nvec + q] = v;
        if constexpr (kTab)
          Obj::map4r(acc, x, d, rtab[j]);
        else if constexpr (!Obj::kNeighbor)
          map4<Obj>(acc, x, 0.f, 4 * q, d);
      }
    }
    if constexpr (Obj::kNeighbor) {
      team_sync(nthr);  // every x' of the row is in the stage
#pragma unroll(VPT <= 2 ? VPT : 2)
      for (int j = 0; j < VPT; ++j) {
        const int q = tid + j * nthr;
        if (q < nvec) map4<Obj>(acc, xdst[q], (q + 1 < nvec) ? xdst[q + 1].x : 0.f, 4 * q, d);
      }
    }
    warp_combine<Obj>(acc);
    if (lane == 0) {
#pragma unroll
      for (int j = 0; j < Obj::kAcc; ++j) red[s][warp * Obj::kAcc + j] = acc[j];
    }
    fence_proxy_async_shared();  // x', v' visible to the bulk stores
    __syncwarp();
    if (lane == 0) mbar_arrive(&done[s]);
    if (++s == stages) {
      s = 0;
      ph ^= 1u;
    }
  }
}

// ------------------------------------------------- step kernel: cluster (wide rows)
// NEXT-3 within one GPU (the paper's "tile matrix" split, applied to a
// row): a thread-block cluster of C CTAs owns a row at a time, CTA k the
// column block [k chunk, (k+1) chunk) of float4s.  Each CTA is a k_step_tma
// pipeline on its block (producer / compute / finaliser warps, bulk copies of
// the block of x, v, pb, G and bounds).  Per row the C finalisers publish
// their block partial (and, for neighbour functors, the block's first and
// last x') into CTA 0's shared memory (DSMEM stores + remote mbarrier
// arrivals); CTA 0 combines the blocks in rank order, adds the terms that
// straddle block boundaries, decides the pbest update and sends the decision
// back to every CTA, which then bulk-stores its block of x', v' (and pb).
template <class Obj, int VPT, bool kB>
__global__ void __launch_bounds__(kMaxThreadsCluster + 64, 1)
    k_step_cluster(const __grid_constant__ SwarmArgs a, int stages, int C, int chunk) {
  extern __shared__ __align__(128) unsigned char dsmem[];
  constexpr int kSlot = Obj::kAcc + 2;  // partial accumulators, first x', last x'
  const int nvec = a.nvec, d = a.d;
  const int nthr = (int)blockDim.x - 64;
  const int nwarps = nthr >> 5;
  const int crank = (int)cluster_rank();
  const int cid = blockIdx.x / C, ncl = gridDim.x / C;
  const int q0 = crank * chunk;
  const int cnt = max(0, min(chunk, nvec - q0));  // float4s of this CTA's block
  const bool row_tail = q0 + cnt < nvec;            // a later block follows
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float4* sB = sG + chunk;
  float4* ring = sB + (kB ? 4 * chunk : 0);
  __shared__ float red[kClusterStages][(kMaxThreadsCluster / 32) * 2];
  // CTA 0: per rank {acc0, acc1, first x', last x'}; every CTA: {improved, f}.
  // Both arrive by st.async, which signals the receiver's mbarrier (complete_tx).
  __shared__ __align__(16) float4 parts[kClusterStages][16];
  __shared__ __align__(8) float2 dec[kClusterStages];
  __shared__ unsigned long long full[kClusterStages], empty[kClusterStages], done[kClusterStages];
  __shared__ unsigned long long pbar[kClusterStages], dbar[kClusterStages], gbar;
  __shared__ unsigned long long s_inc;  // incumbent of this iteration (after the exchange merge)
  __shared__ int s_src;
  __shared__ int sflag[kClusterStages];     // lazy pbest: the stage's row had PB == X
  // Row schedule: CTA 0's producer picks the cluster's rows (round robin over
  // clusters, or claimed from ctl->row_claim as in k_step_tma) and sends each
  // stage's {row, lazy flag} to every CTA of the cluster (st.async + rbar);
  // a CTA's producer copies it to srow / sflag for its own warps.
  __shared__ __align__(8) float2 rmsg[kClusterStages];  // {row bits, flag bits; flag -1: no more rows}
  __shared__ unsigned long long rbar[kClusterStages];
  __shared__ long long srow[kClusterStages];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    mbar_init(&gbar, 1);
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&done[s], (unsigned)nwarps);
      mbar_init(&empty[s], 1);
      mbar_init(&pbar[s], 1);
      mbar_init(&dbar[s], 1);
      mbar_init(&rbar[s], 1);
    }
    mbar_fence_init();
  }
  __syncthreads();
  cluster_sync_all();  // every CTA's barriers exist before any remote arrival
  pdl_wait_and_release();
  const uint32_t t = a.ctl->t + 1u;
  const unsigned blk_bytes = (unsigned)cnt * 16u;

  if (warp == nwarps) {  // ---------------- producer
    int xsrc = -1;
    unsigned long long xinc = 0;
    if (a.exchange) xinc = exchange_merge_warp(a, merge_iter(a, t), lane, &xsrc);  // the all-gather's merge
    if (lane == 0) {
      const float* gsrc = a.G;
      s_src = -1;
      s_inc = a.ctl->key_cur;
      if (a.exchange) {
        s_inc = xinc;
        s_src = xsrc;
        gsrc = merged_gbest_row(a, merge_iter(a, t), xsrc);
      }
      mbar_expect_tx(&gbar, blk_bytes * (kB ? 5u : 1u));  // releases s_inc / s_src too
      if (cnt > 0) {
        bulk_g2s(sG, gsrc + (size_t)q0 * 4, blk_bytes, &gbar);
        if (kB)
          for (int k = 0; k < 4; ++k)
            bulk_g2s(sB + k * chunk, a.bounds + ((size_t)k * nvec + q0) * 4, blk_bytes, &gbar);
      }
      int s = 0;
      unsigned ph = 0;
      int k = 0;
      const long long n = a.n_local;
      const long long pd = (long long)a.l2pf * ncl;  // L2 prefetch, as in k_step_tma
      // CTA 0 only: the claim front (k_step_tma's scheme, per cluster)
      // (dynamic claims measured slower here -- W16K 808 -> 885-904 us -- so
      // they are opt-in: dyn_rows bit 1)
      unsigned long long* claim_ctr = &a.ctl->row_claim;
      const bool dyn = (a.dyn_rows & 2) != 0;
      long long i = cid, i_next = 0;
      int fl_next = 0, pfl_next = 0;
      if (crank == 0) {
        i_next = i >= n ? n : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + ncl : i + ncl);
        fl_next = (a.lazy_pb && i < n) ? a.pbx[i] : 0;
        pfl_next = (pd && i + pd < n) ? a.pbx[i + pd] : 0;
      }
      for (;; ++k) {
        if (k >= stages) mbar_wait(&empty[s], ph ^ 1u);
        if (crank == 0) {  // pick the row, send {row, flag} to every CTA of the cluster
          long long r = -1;
          int fl = -1;
          if (i < n) {
            r = i;
            fl = fl_next;
            const long long i_nn = i_next >= n ? n
                                   : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + ncl
                                          : i_next + ncl);
            if (a.lazy_pb && i_next < n) fl_next = a.pbx[i_next];
            if (pd && i + pd < n) {
              const int pfl = pfl_next;
              if (i_next + pd < n) pfl_next = a.pbx[i_next + pd];
              if (pfl || a.l2pf_all) {  // the whole row (every CTA's block)
                const size_t po = (size_t)(i + pd) * nvec * 4;
                const unsigned rb = (unsigned)nvec * 16u;
                bulk_prefetch_l2(a.X + po, rb);
                bulk_prefetch_l2(a.V + po, rb);
                if (!pfl) bulk_prefetch_l2(a.PB + po, rb);
              }
            }
            i = i_next;
            i_next = i_nn;
          }
          const float2 m = make_float2(__int_as_float((int)r), __int_as_float(fl));
          for (int c = 0; c < C; ++c) st_async_v2(map_to_rank(&rmsg[s], c), m, map_to_rank(&rbar[s], c));
        }
        mbar_expect_tx(&rbar[s], 8u);
        mbar_wait_cluster(&rbar[s], ph);
        const float2 m = rmsg[s];
        const int fl = __float_as_int(m.y);
        if (fl < 0) {  // sentinel: the compute warps and the finaliser stop here
          srow[s] = -1;
          mbar_arrive(&full[s]);
          break;
        }
        const long long r = __float_as_int(m.x);
        float4* st = ring + (size_t)s * 3 * chunk;
        PSO_DCHECK(r >= 0 && r < n && s < stages && stages <= kMaxStages && q0 + cnt <= nvec);
        PSO_DCHECK((size_t)((const unsigned char*)(st + 3 * chunk) - dsmem) <= dyn_smem_bytes());
        sflag[s] = fl;
        srow[s] = r;
        mbar_expect_tx(&full[s], (fl ? 2u : 3u) * blk_bytes);  // releases sflag[s], srow[s] too
        if (cnt > 0) {
          const size_t off = ((size_t)r * nvec + q0) * 4;
          bulk_g2s(st, a.X + off, blk_bytes, &full[s]);
          bulk_g2s(st + chunk, a.V + off, blk_bytes, &full[s]);
          if (!fl) bulk_g2s(st + 2 * chunk, a.PB + off, blk_bytes, &full[s]);
        }
        if (++s == stages) {
          s = 0;
          ph ^= 1u;
        }
      }
    }
    return;
  }

  if (warp == nwarps + 1) {  // ---------------- finaliser
    __shared__ int s_last;
    if (lane == 0) {
      mbar_wait(&gbar, 0);
      const uint32_t inc_ord = (uint32_t)(s_inc >> 32);
      unsigned long long best = ~0ull;
      unsigned nimp = 0, n_pbl = 0, n_pbs = 0;
      int s = 0, prev = -1;
      unsigned ph = 0;
      for (;;) {
        mbar_wait(&full[s], ph);
        const long long r = srow[s];
        if (r < 0) break;
        const uint32_t gi = (uint32_t)(a.row_begin + r);
        const float pf_old = crank == 0 ? a.pf[r] : 0.f;
        mbar_wait(&done[s], ph);
        float c[Obj::kAcc];
        Obj::init(c);
        for (int w = 0; w < nwarps; ++w) {
          float b[Obj::kAcc];
#pragma unroll
          for (int j = 0; j < Obj::kAcc; ++j) b[j] = red[s][w * Obj::kAcc + j];
          Obj::combine(c, b);
        }
        const float4* st = ring + (size_t)s * 3 * chunk;
        const int fl = sflag[s];
        const float4* xnew = fl ? st + 2 * chunk : st;  // where the compute warps put x'
        // publish {partial, first x', last x'} to CTA 0 (one 16-byte st.async)
        {
          float4 msg = make_float4(c[0], Obj::kAcc > 1 ? c[Obj::kAcc - 1] : 0.f, 0.f, 0.f);
          if (Obj::kNeighbor && cnt > 0) {
            msg.z = xnew[0].x;
            msg.w = xnew[cnt - 1].w;
          }
          st_async_v4(map_to_rank(&parts[s][crank], 0), msg, map_to_rank(&pbar[s], 0));
        }
        mbar_expect_tx(&dbar[s], 8u);  // this CTA's decision message
        if (crank == 0) {  // combine blocks in rank order, decide, broadcast
          mbar_expect_tx(&pbar[s], 16u * (unsigned)C);
          mbar_wait_cluster(&pbar[s], ph);
          float tot[Obj::kAcc];
          Obj::init(tot);
          for (int k = 0; k < C; ++k) {
            const float4 pk = parts[s][k];
            float ck_acc[2] = {pk.x, pk.y};
            Obj::combine(tot, ck_acc);
            const int qk = k * chunk, ck = min(chunk, nvec - qk);
            if (Obj::kNeighbor && k + 1 < C && ck > 0 && qk + ck < nvec) {
              float bterm[Obj::kAcc];
              Obj::init(bterm);
              const int jl = 4 * (qk + ck) - 1;  // last dim of block k
              Obj::map(bterm, pk.w, parts[s][k + 1].z, jl, d);
              Obj::combine(tot, bterm);
            }
          }
          const float f = Obj::finalize(tot, d);
          const float imp = (f < pf_old) ? 1.f : 0.f;  // strict; NaN never improves
          for (int k = 0; k < C; ++k)
            st_async_v2(map_to_rank(&dec[s], k), make_float2(imp, f), map_to_rank(&dbar[s], k));
          if (imp != 0.f) {
            a.pf[r] = f;
            ++nimp;
          }
          if (a.lazy_pb && (int)(imp != 0.f) != fl) a.pbx[r] = imp != 0.f ? 1 : 0;
          n_pbl += fl ? 0u : 1u;
          n_pbs += (a.lazy_pb ? (fl && imp == 0.f) : (imp != 0.f)) ? 1u : 0u;
          if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf
            const unsigned long long key = pack_key(f, gi);
            best = key < best ? key : best;
          }
        }
        mbar_wait_cluster(&dbar[s], ph);
        const bool improved = dec[s].x != 0.f;
        if (cnt > 0) {
          const size_t off = ((size_t)r * nvec + q0) * 4;
          bulk_s2g(a.X + off, xnew, blk_bytes);
          bulk_s2g(a.V + off, st + chunk, blk_bytes);
          if (!a.lazy_pb) {
            if (improved) bulk_s2g(a.PB + off, st, blk_bytes);
          } else if (fl && !improved) {
            bulk_s2g(a.PB + off, st, blk_bytes);  // deferred copy of the old x
          }
        }
        bulk_commit();
        if (prev >= 0) {
          bulk_wait_read<1>();
          mbar_arrive(&empty[prev]);
        }
        prev = s;
        if (++s == stages) {
          s = 0;
          ph ^= 1u;
        }
      }
      bulk_wait_all();
      fence_proxy_async_global();
      if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
      if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
      if (n_pbl) atomicAdd(&a.ctl->pb_loads, (unsigned long long)n_pbl);
      if (n_pbs) atomicAdd(&a.ctl->pb_stores, (unsigned long long)n_pbs);
      __threadfence();
      s_last = (atomicAdd(&a.ctl->done, 1u) == gridDim.x - 1) ? 1 : 0;
      if (s_last) a.ctl->row_claim = 0;  // every cluster's claims are done (see the producer)
    }
    __syncwarp();
    if (s_last) warp_gbest_epilogue(a, t, lane, s_inc, s_src);
    return;
  }

  // ---------------- compute warps
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  mbar_wait(&gbar, 0);
  int s = 0;
  unsigned ph = 0;
  for (;;) {
    float4* st = ring + (size_t)s * 3 * chunk;
    mbar_wait(&full[s], ph);
    const long long r = srow[s];
    if (r < 0) break;
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    const int fl = sflag[s];
    float4* xdst = fl ? st + 2 * chunk : st;
    float acc[Obj::kAcc];
    Obj::init(acc);
#pragma unroll(VPT <= 2 ? VPT : 2)
    for (int j = 0; j < VPT; ++j) {
      const int ql = tid + j * nthr;
      if (ql < cnt) {
        const int q = q0 + ql;
        float4 x = st[ql], v = st[chunk + ql];
        const float4 g = sG[ql];
        move4_draw<kB>(mp, key, t, gi, (uint32_t)q, fl, x, v, st + 2 * chunk + ql, g, sB, chunk, ql);
        if ((d & 3) && q == nvec - 1) {
          const int jj = 4 * q;
          if (jj + 1 >= d) x.y = v.y = 0.f;
          if (jj + 2 >= d) x.z = v.z = 0.f;
          if (jj + 3 >= d) x.w = v.w = 0.f;
        }
        xdst[ql] = x;
        st[chunk + ql] = v;
        if constexpr (!Obj::kNeighbor) map4<Obj>(acc, x, 0.f, 4 * q, d);
      }
    }
    if constexpr (Obj::kNeighbor) {
      team_sync(nthr);  // every x' of the block is in the stage
#pragma unroll(VPT <= 2 ? VPT : 2)
      for (int j = 0; j < VPT; ++j) {
        const int ql = tid + j * nthr;
        if (ql < cnt) {
          const int q = q0 + ql;
          const float4 x = xdst[ql];
          if (ql + 1 < cnt) {
            map4<Obj>(acc, x, xdst[ql + 1].x, 4 * q, d);
          } else if (!row_tail) {
            map4<Obj>(acc, x, 0.f, 4 * q, d);  // the row's last float4
          } else {  // x_{j+1} of the last dim lives in the next block: CTA 0 adds it
            Obj::map(acc, x.x, x.y, 4 * q, d);
            Obj::map(acc, x.y, x.z, 4 * q + 1, d);
            Obj::map(acc, x.z, x.w, 4 * q + 2, d);
          }
        }
      }
    }
    warp_combine<Obj>(acc);
    if (lane == 0) {
#pragma unroll
      for (int j = 0; j < Obj::kAcc; ++j) red[s][warp * Obj::kAcc + j] = acc[j];
    }
    fence_proxy_async_shared();
    __syncwarp();
    if (lane == 0) mbar_arrive(&done[s]);
    if (++s == stages) {
      s = 0;
      ph ^= 1u;
    }
  }
}

// ------------------------------------------------- resident kernel (small swarms)
// NEXT-1 latency path: for tiny swarms (d <= 128, n d <= 8192)
// one CTA keeps X, V, PB, pf and G in shared memory for all `iters`
// iterations of a pso_step call, with one __syncthreads pair per iteration
// instead of a kernel launch.  Rows are packed into warps in lane groups of
// gs = pow2ceil(nvec) lanes (lane q of a group owns float4 q).  The per-row
// reduction is the xor butterfly over the group, which is exactly the order
// k_step_reg's one-warp shape produces for these rows (its wider butterfly
// steps only add the identities of idle lanes), so fitness, decisions and
// state are bitwise those of the streaming kernels.
template <class Obj, bool kB>
__global__ void __launch_bounds__(1024, 1) k_resident(const __grid_constant__ SwarmArgs a, int iters) {
  extern __shared__ __align__(16) unsigned char dsmem[];
  const int nvec = a.nvec, d = a.d;
  const int n = (int)a.n_local;
  const int cells = n * nvec;
  float4* sX = reinterpret_cast<float4*>(dsmem);
  float4* sV = sX + cells;
  float4* sP = sV + cells;
  float4* sG = sP + cells;
  float4* sB = sG + nvec;  // kB: [vlo | vhi | xlo | xhi]
  float* spf = reinterpret_cast<float*>(sB + (kB ? 4 * nvec : 0));
  __shared__ unsigned long long s_acc;
  __shared__ unsigned s_imp;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = blockDim.x >> 5;
  int gs = 1;
  while (gs < nvec) gs <<= 1;
  const int rpw = 32 / gs;              // rows per warp pass
  const int sub = lane & (gs - 1);      // float4 index within the row
  const int leader = lane & ~(gs - 1);  // lane holding the row's result
  const float4* X4 = reinterpret_cast<const float4*>(a.X);
  const float4* V4 = reinterpret_cast<const float4*>(a.V);
  const float4* P4 = reinterpret_cast<const float4*>(a.PB);
  for (int i = tid; i < cells; i += blockDim.x) {
    sX[i] = X4[i];
    sV[i] = V4[i];
    sP[i] = P4[i];
  }
  for (int i = tid; i < nvec; i += blockDim.x) sG[i] = reinterpret_cast<const float4*>(a.G)[i];
  if (kB)
    for (int i = tid; i < 4 * nvec; i += blockDim.x)
      sB[i] = reinterpret_cast<const float4*>(a.bounds)[i];
  for (int i = tid; i < n; i += blockDim.x) spf[i] = a.pf[i];
  const unsigned long long cur0 = a.ctl->key_cur;
  const uint32_t t0 = a.ctl->t;
  if (tid == 0) {
    s_acc = cur0;
    s_imp = 0;
  }
  __syncthreads();
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  unsigned long long cur = cur0;
  for (int it = 0; it < iters; ++it) {
    const uint32_t t = t0 + 1u + (uint32_t)it;
    const uint32_t inc_ord = (uint32_t)(cur >> 32);
    unsigned long long best = ~0ull;
    unsigned nimp = 0;
    for (int base = warp * rpw; base < n; base += nwarps * rpw) {  // warp-uniform loop
      const int r = base + (lane / gs);
      const bool row_ok = r < n;
      const bool act = row_ok && sub < nvec;
      const uint32_t gi = (uint32_t)(a.row_begin + r);
      const int c = r * nvec + sub;
      float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
      if (act) {
        float4 v = sV[c];
        const float4 pb = sP[c], g = sG[sub];
        x = sX[c];
        const float4 r1 = raw24x4(key, kTagR1, t, gi, (uint32_t)sub);
        const float4 r2 = raw24x4(key, kTagR2, t, gi, (uint32_t)sub);
        move4<kB>(mp, x, v, pb, g, r1, r2, sB, nvec, sub);
        if ((d & 3) && sub == nvec - 1) {
          const int jj = 4 * sub;
          if (jj + 1 >= d) x.y = v.y = 0.f;
          if (jj + 2 >= d) x.z = v.z = 0.f;
          if (jj + 3 >= d) x.w = v.w = 0.f;
        }
        sX[c] = x;
        sV[c] = v;
      }
      float acc[Obj::kAcc];
      Obj::init(acc);
      float nx = 0.f;
      if constexpr (Obj::kNeighbor) {
        nx = __shfl_down_sync(kFull, x.x, 1);
        if (sub + 1 >= nvec) nx = 0.f;
      }
      if (act) map4<Obj>(acc, x, nx, 4 * sub, d);
      for (int off = gs >> 1; off > 0; off >>= 1) {
        float o[Obj::kAcc];
#pragma unroll
        for (int k = 0; k < Obj::kAcc; ++k) o[k] = __shfl_xor_sync(kFull, acc[k], off);
        Obj::combine(acc, o);
      }
      const float f = Obj::finalize(acc, d);
      const int imp_l = (row_ok && lane == leader && f < spf[r]) ? 1 : 0;  // strict
      const bool improved = __shfl_sync(kFull, imp_l, leader) != 0;
      __syncwarp();
      if (improved) {
        if (act) sP[c] = x;
        if (lane == leader) {
          spf[r] = f;
          ++nimp;
        }
      }
      if (row_ok && lane == leader && f == f && ord_f32(f) < inc_ord) {
        const unsigned long long k = pack_key(f, gi);
        best = k < best ? k : best;
      }
    }
    for (int off = 16; off > 0; off >>= 1) {
      const unsigned long long o = __shfl_xor_sync(kFull, best, off);
      best = o < best ? o : best;
      nimp += __shfl_xor_sync(kFull, nimp, off);
    }
    if (lane == 0) {
      if (best != ~0ull) atomicMin(&s_acc, best);
      if (nimp) atomicAdd(&s_imp, nimp);
    }
    __syncthreads();
    const unsigned long long acc_k = s_acc;
    if (acc_k < cur) {
      const int lr = (int)((long long)(uint32_t)acc_k - a.row_begin);
      for (int q = tid; q < nvec; q += blockDim.x) sG[q] = sP[lr * nvec + q];
      cur = acc_k;
    }
    __syncthreads();
  }
  float4* X4w = reinterpret_cast<float4*>(a.X);
  float4* V4w = reinterpret_cast<float4*>(a.V);
  float4* P4w = reinterpret_cast<float4*>(a.PB);
  for (int i = tid; i < cells; i += blockDim.x) {
    X4w[i] = sX[i];
    V4w[i] = sV[i];
    P4w[i] = sP[i];
  }
  for (int i = tid; i < nvec; i += blockDim.x) reinterpret_cast<float4*>(a.G)[i] = sG[i];
  for (int i = tid; i < n; i += blockDim.x) a.pf[i] = spf[i];
  if (tid == 0) {
    a.ctl->key_cur = cur;
    a.ctl->key_acc = cur;
    a.ctl->t = t0 + (uint32_t)iters;
    a.ctl->improvements += s_imp;
  }
}

// ------------------------------------------------- grid-resident kernel
// NEXT-1 for mid-size swarms whose state fits in the GPU's aggregate shared
// memory (e.g. C2, 1024 x 1000 = 12 MB): a cooperative persistent grid; CTA b
// owns rows b, b + grid, ... and keeps their x, v, pb (and pf) in shared
// memory for all `iters` iterations of a pso_step call, so an iteration moves
// no row data through L2/HBM at all.  Per row the arithmetic and the
// reduction order are k_step_tma's (thread-sequential over its float4s, warp
// butterfly, warps combined in index order by one thread), so results are
// bitwise those of the streaming kernel (rows are processed in pairs, each
// with its own accumulators).  Per iteration: each CTA publishes its best
// candidate row to cand[parity][cta] and its key to cand_key[parity][cta]; a
// grid barrier (acq_rel atomic ticket + release of a generation flag); then
// every CTA folds all keys itself and pulls the winner's row into its
// shared-memory G.
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned atom_add_acq_rel_u32(unsigned* p, unsigned v) {
  unsigned o;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(o) : "l"(p), "r"(v) : "memory");
  return o;
}

template <class Obj, int VPT, bool kB>
__global__ void __launch_bounds__(kMaxThreadsWide, 1) k_gridres(const __grid_constant__ SwarmArgs a, int iters) {
  extern __shared__ __align__(16) unsigned char dsmem[];
  const int nvec = a.nvec, d = a.d;
  const int nthr = blockDim.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nwarps = nthr >> 5;
  const int grid = gridDim.x, b = blockIdx.x;
  const long long n = a.n_local;
  const int myrows = (int)((n - b + grid - 1) / grid);  // rows b, b+grid, ...
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float4* sB = sG + nvec;                          // kB: [vlo | vhi | xlo | xhi]
  float4* sRows = sB + (kB ? 4 * nvec : 0);        // [myrows][3][nvec]
  float* spf = reinterpret_cast<float*>(sRows + (size_t)myrows * 3 * nvec);
  __shared__ float red[2 * (kMaxThreadsWide / 32) * 2];  // [row of the pair][warp][acc]
  __shared__ float s_f2[2];
  __shared__ int s_imp2[2];
  __shared__ unsigned long long s_best;
  __shared__ int s_best_row;
  __shared__ unsigned long long s_kmin[kMaxThreadsWide / 32];

  // ---- load this CTA's rows and G
  for (int k = 0; k < myrows; ++k) {
    const long long r = b + (long long)k * grid;
    const float4* X4 = reinterpret_cast<const float4*>(a.X) + r * nvec;
    const float4* V4 = reinterpret_cast<const float4*>(a.V) + r * nvec;
    const float4* P4 = reinterpret_cast<const float4*>(a.PB) + r * nvec;
    float4* st = sRows + (size_t)k * 3 * nvec;
    for (int q = tid; q < nvec; q += nthr) {
      st[q] = X4[q];
      st[nvec + q] = V4[q];
      st[2 * nvec + q] = P4[q];
    }
    if (tid == 0) spf[k] = a.pf[r];
  }
  for (int q = tid; q < nvec; q += nthr) sG[q] = reinterpret_cast<const float4*>(a.G)[q];
  if (kB)
    for (int q = tid; q < 4 * nvec; q += nthr) sB[q] = reinterpret_cast<const float4*>(a.bounds)[q];
  const unsigned long long cur0 = a.ctl->key_cur;
  const uint32_t t0 = a.ctl->t;
  __syncthreads();

  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  unsigned long long cur = cur0;
  unsigned nimp = 0;
  unsigned long long* ckey = a.cand_key;  // [2 parities][grid] candidate keys
  const unsigned gen0 = ld_acquire_u32(&a.ctl->bar_gen);  // barrier `it` completes at gen0 + it + 1
  // Overlap (VPT <= 2): while the grid barrier of iteration t settles, every
  // thread already computes the gbest-free part of iteration t + 1 for the
  // CTA's first row pair -- both Philox draws and ab = w v + (c1 r1)(pb - x)
  // -- and keeps it in registers; after the barrier only (c2 r2)(g - x), the
  // clamps and the move remain.  Same operations in the same order.
  constexpr bool kOverlap = VPT <= 2;
  float4 pre_ab[2][kOverlap ? VPT : 1], pre_m2[2][kOverlap ? VPT : 1];
  bool have_pre = false;
  for (int it = 0; it < iters; ++it) {
    const uint32_t t = t0 + 1u + (uint32_t)it;
    const int par = (int)(t & 1u);
    const uint32_t inc_ord = (uint32_t)(cur >> 32);
    unsigned long long best = ~0ull;
    int best_row = -1;
    // Rows in pairs: both rows' updates and maps in one pass (twice the
    // independent work per thread), one reduction barrier for the pair.  Per
    // row the operation order is unchanged (bitwise k_step_tma).
    for (int k0 = 0; k0 < myrows; k0 += 2) {
      const int nk = (myrows - k0) < 2 ? (myrows - k0) : 2;
      const bool use_pre = kOverlap && have_pre && k0 == 0;
      float acc[2][Obj::kAcc];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        Obj::init(acc[u]);
        if (u < nk) {
          const int k = k0 + u;
          const uint32_t gi = (uint32_t)(a.row_begin + b + (long long)k * grid);
          float4* st = sRows + (size_t)k * 3 * nvec;
#pragma unroll(VPT <= 2 ? VPT : 2)
          for (int j = 0; j < VPT; ++j) {
            const int q = tid + j * nthr;
            if (q < nvec) {
              float4 x = st[q], v = st[nvec + q];
              const float4 g = sG[q];
              if constexpr (kOverlap) {
                if (use_pre) {
                  move_post4<kB>(mp, x, v, g, pre_m2[u][j], pre_ab[u][j], sB, nvec, q);
                } else {
                  const float4 pb = st[2 * nvec + q];
                  const float4 r1 = raw24x4(key, kTagR1, t, gi, (uint32_t)q);
                  const float4 r2 = raw24x4(key, kTagR2, t, gi, (uint32_t)q);
                  move4<kB>(mp, x, v, pb, g, r1, r2, sB, nvec, q);
                }
              } else {
                const float4 pb = st[2 * nvec + q];
                const float4 r1 = raw24x4(key, kTagR1, t, gi, (uint32_t)q);
                const float4 r2 = raw24x4(key, kTagR2, t, gi, (uint32_t)q);
                move4<kB>(mp, x, v, pb, g, r1, r2, sB, nvec, q);
              }
              if ((d & 3) && q == nvec - 1) {
                const int jj = 4 * q;
                if (jj + 1 >= d) x.y = v.y = 0.f;
                if (jj + 2 >= d) x.z = v.z = 0.f;
                if (jj + 3 >= d) x.w = v.w = 0.f;
              }
              st[q] = x;
              st[nvec + q] = v;
              if constexpr (!Obj::kNeighbor) map4<Obj>(acc[u], x, 0.f, 4 * q, d);
            }
          }
        }
      }
      if constexpr (Obj::kNeighbor) {
        __syncthreads();
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          if (u < nk) {
            const float4* st = sRows + (size_t)(k0 + u) * 3 * nvec;
#pragma unroll(VPT <= 2 ? VPT : 2)
            for (int j = 0; j < VPT; ++j) {
              const int q = tid + j * nthr;
              if (q < nvec) map4<Obj>(acc[u], st[q], (q + 1 < nvec) ? st[q + 1].x : 0.f, 4 * q, d);
            }
          }
        }
      }
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        if (u < nk) {
          warp_combine<Obj>(acc[u]);
          if (lane == 0) {
#pragma unroll
            for (int j = 0; j < Obj::kAcc; ++j) red[(u * nwarps + warp) * Obj::kAcc + j] = acc[u][j];
          }
        }
      }
      __syncthreads();
      if (tid < nk) {  // thread u finalises row k0 + u (warps combined in index order)
        const int u = tid, k = k0 + u;
        float c[Obj::kAcc];
        Obj::init(c);
        for (int w = 0; w < nwarps; ++w) {
          float o[Obj::kAcc];
#pragma unroll
          for (int j = 0; j < Obj::kAcc; ++j) o[j] = red[(u * nwarps + w) * Obj::kAcc + j];
          Obj::combine(c, o);
        }
        const float f = Obj::finalize(c, d);
        const int imp = (f < spf[k]) ? 1 : 0;  // strict; NaN never improves
        if (imp) spf[k] = f;
        s_imp2[u] = imp;
        s_f2[u] = f;
      }
      __syncthreads();
      if (tid == 0) {  // gbest candidates in row order (equal keys: the lower global index)
        for (int u = 0; u < nk; ++u) {
          const float f = s_f2[u];
          nimp += (unsigned)s_imp2[u];
          const uint32_t gi = (uint32_t)(a.row_begin + b + (long long)(k0 + u) * grid);
          if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
            const unsigned long long kk = pack_key(f, gi);
            if (kk < best) {
              best = kk;
              best_row = k0 + u;
            }
          }
        }
      }
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        if (u < nk && s_imp2[u]) {  // pbest copy (Alg. 1 lines 7-9)
          float4* st = sRows + (size_t)(k0 + u) * 3 * nvec;
          for (int q = tid; q < nvec; q += nthr) st[2 * nvec + q] = st[q];
        }
      }
      __syncthreads();  // s_imp2 / s_f2 / red are reused by the next pair
    }
    // ---- publish the CTA's candidate (row + key), grid barrier, fold, pull the winner
    if (tid == 0) {
      s_best = best;
      s_best_row = best_row;
    }
    __syncthreads();
    if (s_best_row >= 0) {
      const float4* src = sRows + (size_t)s_best_row * 3 * nvec;  // x' == pb' (it improved)
      float4* dst = reinterpret_cast<float4*>(a.cand) + ((size_t)par * grid + b) * nvec;
      for (int q = tid; q < nvec; q += nthr) dst[q] = src[q];
    }
    if (tid == 0) ckey[(size_t)par * grid + b] = s_best;
    __syncthreads();  // every candidate store of the CTA precedes thread 0's release
    const unsigned gen_done = gen0 + (unsigned)it + 1u;
    bool last = false;
    if (tid == 0) {  // arrival: acq_rel ticket; the last CTA releases the generation
      last = atom_add_acq_rel_u32(&a.ctl->bar_count, 1u) == (unsigned)grid - 1;
      if (last) {
        a.ctl->bar_count = 0;
        st_release_u32(&a.ctl->bar_gen, gen_done);
      }
    }
    // the gbest-free part of the next iteration while the barrier settles
    have_pre = false;
    if constexpr (kOverlap) {
      if (it + 1 < iters) {
        const uint32_t tn = t + 1u;
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          if (u < myrows) {
            const uint32_t gi = (uint32_t)(a.row_begin + b + (long long)u * grid);
            const float4* st = sRows + (size_t)u * 3 * nvec;
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
              const int q = tid + j * nthr;
              if (q < nvec) {
                const float4 r1 = raw24x4(key, kTagR1, tn, gi, (uint32_t)q);
                pre_m2[u][j] = raw24x4(key, kTagR2, tn, gi, (uint32_t)q);
                move_pre4<kB>(mp, st[q], st[nvec + q], st[2 * nvec + q], r1, pre_ab[u][j]);
              }
            }
          }
        }
        have_pre = true;
      }
    }
    if (tid == 0 && !last) {
      while (ld_acquire_u32(&a.ctl->bar_gen) != gen_done) {
      }
    }
    __syncthreads();
    // every CTA folds all candidate keys itself (one parallel L2 read instead
    // of a serial fold by the last arriver); keys of this parity are
    // rewritten only after the next barrier, which every CTA passes after
    // this read
    unsigned long long m = ~0ull;
    const unsigned long long* keys = ckey + (size_t)par * grid;
    for (int c0 = tid; c0 < grid; c0 += 8 * nthr) {  // 8 independent loads in flight per thread
      unsigned long long kk[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int c = c0 + i * nthr;
        kk[i] = c < grid ? __ldcg(keys + c) : ~0ull;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) m = kk[i] < m ? kk[i] : m;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      const unsigned long long o = __shfl_xor_sync(kFull, m, off);
      m = o < m ? o : m;
    }
    if (lane == 0) s_kmin[warp] = m;
    __syncthreads();
    unsigned long long win = ~0ull;
    for (int w = 0; w < nwarps; ++w) win = s_kmin[w] < win ? s_kmin[w] : win;
    if (win < cur) {  // strictly better than the incumbent (candidates already are)
      const long long wr = (long long)(uint32_t)win - a.row_begin;
      const int owner = (int)(wr % grid);
      const float4* src = reinterpret_cast<const float4*>(a.cand) + ((size_t)par * grid + owner) * nvec;
      for (int q = tid; q < nvec; q += nthr) sG[q] = __ldcg(src + q);
      cur = win;
    }
    __syncthreads();
  }

  // ---- write back
  for (int k = 0; k < myrows; ++k) {
    const long long r = b + (long long)k * grid;
    float4* X4 = reinterpret_cast<float4*>(a.X) + r * nvec;
    float4* V4 = reinterpret_cast<float4*>(a.V) + r * nvec;
    float4* P4 = reinterpret_cast<float4*>(a.PB) + r * nvec;
    const float4* st = sRows + (size_t)k * 3 * nvec;
    for (int q = tid; q < nvec; q += nthr) {
      X4[q] = st[q];
      V4[q] = st[nvec + q];
      P4[q] = st[2 * nvec + q];
    }
    if (tid == 0) a.pf[r] = spf[k];
  }
  if (tid == 0 && nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
  if (b == 0) {
    for (int q = tid; q < nvec; q += nthr) reinterpret_cast<float4*>(a.G)[q] = sG[q];
    if (tid == 0) {
      a.ctl->key_cur = cur;
      a.ctl->key_acc = cur;
      a.ctl->t = t0 + (uint32_t)iters;
    }
  }
}

// ------------------------------------------------------------ init kernel
// Alg. 1 lines 1-3 (Sec 3.1): x0 = clamp(xlo + (xhi - xlo) U, xlo, xhi), v0 =
// vlo + (vhi - vlo) U from the X0 / V0 streams at t = 0 (scalar bounds: xlo =
// lo, xhi = hi, vlo = -vmax, vhi = vmax); f = F(x0); pf = f (NaN -> +inf);
// PB = x0; every row is a gbest candidate (key_cur = ~0 on entry).  Thread t
// handles float4 t, t + nthr, ... of a row (any d; the same accumulation
// order as the register kernels); a neighbour functor's x_{j+1} across a
// float4 boundary is recomputed from its Philox word.
// init_float4_at: dims 4 qg .. 4 qg + 3 of the row (qg: global float4 index,
// the Philox counter and the padding test), bounds from float4 qb of a table
// with `bstride` float4 per array (the column split keeps only its block).
template <class K>
__device__ __forceinline__ void init_float4_at(const SwarmArgs& a, const K& key, uint32_t gi,
                                               int qg, const float4* B4, int bstride, int qb,
                                               float4& xo, float4& vo) {
  const int q = qg, d = a.d;
  const float4 ux = uniforms4(key, kTagX0, 0u, gi, (uint32_t)q);
  const float4 uv = uniforms4(key, kTagV0, 0u, gi, (uint32_t)q);
  float xs[4] = {ux.x, ux.y, ux.z, ux.w};
  float vs[4] = {uv.x, uv.y, uv.z, uv.w};
  float4 vlo4 = make_float4(-a.vmax, -a.vmax, -a.vmax, -a.vmax);
  float4 vhi4 = make_float4(a.vmax, a.vmax, a.vmax, a.vmax);
  float4 xlo4 = make_float4(a.lo, a.lo, a.lo, a.lo), xhi4 = make_float4(a.hi, a.hi, a.hi, a.hi);
  if (B4) {
    vlo4 = B4[qb];
    vhi4 = B4[bstride + qb];
    xlo4 = B4[2 * bstride + qb];
    xhi4 = B4[3 * bstride + qb];
  }
  const float vlo[4] = {vlo4.x, vlo4.y, vlo4.z, vlo4.w};
  const float vhi[4] = {vhi4.x, vhi4.y, vhi4.z, vhi4.w};
  const float xlo[4] = {xlo4.x, xlo4.y, xlo4.z, xlo4.w};
  const float xhi[4] = {xhi4.x, xhi4.y, xhi4.z, xhi4.w};
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const bool pad = 4 * q + e >= d;
    const float span = __fsub_rn(xhi[e], xlo[e]);
    const float vspan = __fsub_rn(vhi[e], vlo[e]);
    xs[e] = pad ? 0.f : fminf(fmaxf(__fadd_rn(xlo[e], __fmul_rn(span, xs[e])), xlo[e]), xhi[e]);
    vs[e] = pad ? 0.f : __fadd_rn(vlo[e], __fmul_rn(vspan, vs[e]));
  }
  xo = make_float4(xs[0], xs[1], xs[2], xs[3]);
  vo = make_float4(vs[0], vs[1], vs[2], vs[3]);
}
template <class K>
__device__ __forceinline__ void init_float4(const SwarmArgs& a, const K& key, uint32_t gi, int q,
                                            float4& xo, float4& vo) {
  init_float4_at(a, key, gi, q, reinterpret_cast<const float4*>(a.bounds), a.nvec, q, xo, vo);
}

template <class Obj, int VPT>
__global__ void __launch_bounds__(kMaxThreads, (VPT >= 8) ? 1 : 2)
    k_init(const __grid_constant__ SwarmArgs a) {
  __shared__ RowSmem<Obj> sm;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const PhiloxRoundKeys& key = a.rk;
  const int nvec = a.nvec, d = a.d;
  const uint32_t inc_ord = (uint32_t)(a.ctl->key_cur >> 32);
  unsigned long long best = ~0ull;
  for (long long r = blockIdx.x; r < a.n_local; r += gridDim.x) {
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    float4* Xr = reinterpret_cast<float4*>(a.X) + r * nvec;
    float4* Vr = reinterpret_cast<float4*>(a.V) + r * nvec;
    float4* Pr = reinterpret_cast<float4*>(a.PB) + r * nvec;
    float acc[Obj::kAcc];
    Obj::init(acc);
    for (int q = tid; q < nvec; q += nthr) {
      float4 x, v;
      init_float4(a, key, gi, q, x, v);
      st_stream(Xr + q, x);
      st_stream(Vr + q, v);
      if (!a.lazy_pb) st_stream(Pr + q, x);  // lazy pbest: PB == X is recorded in pbx
      float nx = 0.f;
      if constexpr (Obj::kNeighbor) {
        if (q + 1 < nvec) {
          float4 xn, vn;
          init_float4(a, key, gi, q + 1, xn, vn);
          nx = xn.x;
        }
      }
      map4<Obj>(acc, x, nx, 4 * q, d);
    }
    bool improved;
    float f = cta_fitness<Obj>(acc, sm, d, 0.f, improved, tid, nthr);
    if (tid == 0) {
      if (f != f) f = __int_as_float(0x7f800000);  // reading 11: NaN -> +inf
      a.pf[r] = f;
      if (a.lazy_pb) a.pbx[r] = 1;
      if (ord_f32(f) < inc_ord) {
        const unsigned long long k = pack_key(f, gi);
        best = k < best ? k : best;
      }
    }
  }
  if (cta_finish<Obj>(a, sm, best, 0, tid, nthr)) gbest_epilogue<Obj>(a, sm, 0u, tid, nthr);
}

// ---------------------------------------------------------- debug: objective
// The functor + CTA reduction on given rows (any d; thread t maps float4 t,
// t + nthr, ...).
template <class Obj, int VPT>
__global__ void __launch_bounds__(kMaxThreads) k_eval(const float* X, long long m, int d,
                                                      int nvec, float* out) {
  __shared__ RowSmem<Obj> sm;
  const int tid = threadIdx.x, nthr = blockDim.x;
  for (long long r = blockIdx.x; r < m; r += gridDim.x) {
    const float4* Xr = reinterpret_cast<const float4*>(X) + r * nvec;
    float acc[Obj::kAcc];
    Obj::init(acc);
    for (int q = tid; q < nvec; q += nthr) {
      const float nx = (Obj::kNeighbor && q + 1 < nvec) ? Xr[q + 1].x : 0.f;
      map4<Obj>(acc, Xr[q], nx, 4 * q, d);
    }
    bool improved;
    const float f = cta_fitness<Obj>(acc, sm, d, 0.f, improved, tid, nthr);
    if (tid == 0) out[r] = f;
  }
}

#include "swarm_colsplit.cuh"
#include "swarm_persist.cuh"

template <class Obj>
KernelTable make_kernel_table() {
  KernelTable t{};
  t.neighbor = Obj::kNeighbor;
#define PSO_T(ARR, KER, V, I)                     \
  t.ARR[I][0] = (const void*)KER<Obj, V, false>; \
  t.ARR[I][1] = (const void*)KER<Obj, V, true>;
#define PSO_ALLV(ARR, KER) PSO_T(ARR, KER, 1, 0) PSO_T(ARR, KER, 2, 1) PSO_T(ARR, KER, 4, 2) PSO_T(ARR, KER, 8, 3)
  PSO_ALLV(step_reg, k_step_reg)
  PSO_ALLV(step_tma, k_step_tma)
  t.step_tma_w[1][0] = (const void*)k_step_tma<Obj, 2, false, kMaxThreadsWide>;
  t.step_tma_w[1][1] = (const void*)k_step_tma<Obj, 2, true, kMaxThreadsWide>;
  t.step_tma_w[2][0] = (const void*)k_step_tma<Obj, 4, false, kMaxThreadsWide>;
  t.step_tma_w[2][1] = (const void*)k_step_tma<Obj, 4, true, kMaxThreadsWide>;
  PSO_ALLV(gridres, k_gridres)
  PSO_ALLV(step_cluster, k_step_cluster)
  PSO_ALLV(persist, k_step_persist)
#undef PSO_ALLV
#undef PSO_T
  t.resident[0] = (const void*)k_resident<Obj, false>;
  t.resident[1] = (const void*)k_resident<Obj, true>;
  t.init[0] = (const void*)k_init<Obj, 1>;
  t.init[1] = (const void*)k_init<Obj, 2>;
  t.init[2] = (const void*)k_init<Obj, 4>;
  t.init[3] = (const void*)k_init<Obj, 8>;
  t.eval[0] = (const void*)k_eval<Obj, 1>;
  t.eval[1] = (const void*)k_eval<Obj, 2>;
  t.eval[2] = (const void*)k_eval<Obj, 4>;
  t.eval[3] = (const void*)k_eval<Obj, 8>;
  t.col_step[0] = (const void*)k_col_step<Obj, false>;
  t.col_step[1] = (const void*)k_col_step<Obj, true>;
  t.col_decide = (const void*)k_col_decide<Obj>;
  return t;
}

}  // namespace
}  // namespace fastpso
