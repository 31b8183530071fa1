// swarm_kernels.cu — the fused FastPSO iteration for sm_100a.
//
// One kernel per iteration replaces the paper's five phases (Fig. 5, P:L561-567:
// init / eval / pbest / gbest / swarm) and its materialised random matrices.
// Per particle row (one CTA per row, persistent grid):
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
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"
#include "objectives.cuh"
#include "philox.cuh"

namespace fastpso {
namespace {

constexpr int kMaxThreads = 256;
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

// --- bulk async copy global -> shared (TMA engine) with an mbarrier -------
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count)
               : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
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
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(phase)
      : "memory");
}

// Stage G (nvec float4) into shared memory: one bulk copy issued by thread 0.
__device__ __forceinline__ void stage_gbest(float4* sG, const float* G, int nvec,
                                            unsigned long long* bar) {
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    mbar_expect_tx(bar, (unsigned)nvec * 16u);
    bulk_g2s(sG, G, (unsigned)nvec * 16u, bar);
  }
  __syncthreads();  // barrier initialised before anyone waits on it
}

// --- Eq. 1, 5, 2 on one element, fixed fp32 order, no contraction --------
struct MoveParams {
  float w, c1, c2, lo, hi, vmax;
};
__device__ __forceinline__ void move1(const MoveParams& m, float& x, float& v, float pb, float g,
                                      float r1, float r2) {
  const float a = __fmul_rn(m.w, v);
  const float b = __fmul_rn(__fmul_rn(m.c1, r1), __fsub_rn(pb, x));
  const float c = __fmul_rn(__fmul_rn(m.c2, r2), __fsub_rn(g, x));
  float vn = __fadd_rn(__fadd_rn(a, b), c);
  vn = fminf(fmaxf(vn, -m.vmax), m.vmax);
  x = fminf(fmaxf(__fadd_rn(x, vn), m.lo), m.hi);
  v = vn;
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
  unsigned long long bar;
  int last;
};

// Reduce a[] over the CTA (fixed order: lanes by xor-butterfly, then warps in
// order), finalize in thread 0 and decide the pbest update against pf_old
// (only thread 0's pf_old is read).  Returns f to all threads; *improved is
// the CTA-uniform pbest decision.  Two __syncthreads.
template <class Obj>
__device__ __forceinline__ float cta_fitness(float* a, RowSmem<Obj>& sm, int d, float pf_old,
                                             bool& improved) {
  warp_combine<Obj>(a);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
#pragma unroll
    for (int k = 0; k < Obj::kAcc; ++k) sm.red[warp * Obj::kAcc + k] = a[k];
  }
  __syncthreads();
  if (warp == 0) {
    float c[Obj::kAcc];
    Obj::init(c);
    if (lane < (int)(blockDim.x >> 5)) {
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
  __syncthreads();
  improved = sm.improved != 0;
  return sm.f;
}

// Map the VPT float4 of new positions into the accumulators.  For functors
// that need x_{j+1} the first element of every float4 is published in sFirst.
template <class Obj, int VPT>
__device__ __forceinline__ void map_row(float* acc, const float4 (&x)[VPT], float* sFirst,
                                        int nvec, int d) {
  if constexpr (Obj::kNeighbor) {
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = threadIdx.x + s * blockDim.x;
      if (q < nvec) sFirst[q] = x[s].x;
    }
    __syncthreads();
  }
#pragma unroll
  for (int s = 0; s < VPT; ++s) {
    const int q = threadIdx.x + s * blockDim.x;
    if (q < nvec) {
      const int j = 4 * q;
      float nx = 0.f;
      if constexpr (Obj::kNeighbor) nx = (q + 1 < nvec) ? sFirst[q + 1] : 0.f;
      if (j + 3 < d) {
        Obj::map(acc, x[s].x, x[s].y, j, d);
        Obj::map(acc, x[s].y, x[s].z, j + 1, d);
        Obj::map(acc, x[s].z, x[s].w, j + 2, d);
        Obj::map(acc, x[s].w, nx, j + 3, d);
      } else {  // ragged tail of the row
        if (j < d) Obj::map(acc, x[s].x, x[s].y, j, d);
        if (j + 1 < d) Obj::map(acc, x[s].y, x[s].z, j + 1, d);
        if (j + 2 < d) Obj::map(acc, x[s].z, x[s].w, j + 2, d);
      }
    }
  }
}

// Last-CTA epilogue: publish the iteration's gbest.  world == 1: copy PB[gi]
// into G and advance the incumbent key.  world > 1: write the local candidate
// record (key, PB row) for the all-gather; the select kernel finishes.
__device__ __forceinline__ void gbest_epilogue(const SwarmArgs& a, uint32_t t) {
  __shared__ unsigned long long s_acc, s_cur;
  if (threadIdx.x == 0) {
    __threadfence();
    s_acc = *(volatile unsigned long long*)&a.ctl->key_acc;
    s_cur = a.ctl->key_cur;
  }
  __syncthreads();
  const unsigned long long acc = s_acc, cur = s_cur;
  const bool have = acc < cur;
  const float4* src = nullptr;
  if (have) src = reinterpret_cast<const float4*>(a.PB) +
                  ((long long)(uint32_t)acc - a.row_begin) * a.nvec;
  if (a.world == 1) {
    if (have) {
      float4* G4 = reinterpret_cast<float4*>(a.G);
      for (int q = threadIdx.x; q < a.nvec; q += blockDim.x) G4[q] = __ldcg(src + q);
    }
    if (threadIdx.x == 0) {
      if (have) a.ctl->key_cur = acc;
      a.ctl->t = t;
      a.ctl->done = 0;
    }
  } else {
    unsigned long long* hdr = reinterpret_cast<unsigned long long*>(a.send);
    float4* row = reinterpret_cast<float4*>(a.send + 16);
    if (have)
      for (int q = threadIdx.x; q < a.nvec; q += blockDim.x) row[q] = __ldcg(src + q);
    if (threadIdx.x == 0) {
      hdr[0] = have ? acc : ~0ull;
      hdr[1] = 0;
      a.ctl->t = t;
      a.ctl->done = 0;
    }
  }
}

// Publish this CTA's candidate and improvement count; returns true in the
// last CTA to finish (which then runs gbest_epilogue).
template <class Obj>
__device__ __forceinline__ bool cta_finish(const SwarmArgs& a, RowSmem<Obj>& sm,
                                           unsigned long long best, unsigned nimp) {
  __syncthreads();  // every PB / X / V store of this CTA is issued
  if (threadIdx.x == 0) {
    if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
    if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
    __threadfence();
    const unsigned ticket = atomicAdd(&a.ctl->done, 1u);
    sm.last = (ticket == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  return sm.last != 0;
}

// ------------------------------------------------------------ step kernel
template <class Obj, int VPT>
__global__ void __launch_bounds__(kMaxThreads, (VPT >= 8) ? 1 : 2)
    k_step(const SwarmArgs a) {
  extern __shared__ __align__(16) unsigned char dsmem[];
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float* sFirst = reinterpret_cast<float*>(sG + a.nvec);
  __shared__ RowSmem<Obj> sm;

  stage_gbest(sG, a.G, a.nvec, &sm.bar);
  const uint32_t t = a.ctl->t + 1u;
  const uint32_t inc_ord = (uint32_t)(a.ctl->key_cur >> 32);
  const PhiloxKey key{a.seed_lo, a.seed_hi};
  const MoveParams mp{a.w, a.c1, a.c2, a.lo, a.hi, a.vmax};
  const int nvec = a.nvec, d = a.d;
  const bool ragged = (d & 3) != 0;
  mbar_wait(&sm.bar, 0);

  unsigned long long best = ~0ull;
  unsigned nimp = 0;
  for (long long r = blockIdx.x; r < a.n_local; r += gridDim.x) {
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    float4* Xr = reinterpret_cast<float4*>(a.X) + r * nvec;
    float4* Vr = reinterpret_cast<float4*>(a.V) + r * nvec;
    float4* Pr = reinterpret_cast<float4*>(a.PB) + r * nvec;
    float4 x[VPT], v[VPT], pb[VPT];
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = threadIdx.x + s * blockDim.x;
      if (q < nvec) {
        x[s] = ld_stream(Xr + q);
        v[s] = ld_stream(Vr + q);
        pb[s] = ld_stream(Pr + q);
      }
    }
    const float pf_old = (threadIdx.x == 0) ? a.pf[r] : 0.f;
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = threadIdx.x + s * blockDim.x;
      if (q < nvec) {
        const float4 g = sG[q];
        const float4 r1 = uniforms4(key, kTagR1, t, gi, (uint32_t)q);
        const float4 r2 = uniforms4(key, kTagR2, t, gi, (uint32_t)q);
        move1(mp, x[s].x, v[s].x, pb[s].x, g.x, r1.x, r2.x);
        move1(mp, x[s].y, v[s].y, pb[s].y, g.y, r1.y, r2.y);
        move1(mp, x[s].z, v[s].z, pb[s].z, g.z, r1.z, r2.z);
        move1(mp, x[s].w, v[s].w, pb[s].w, g.w, r1.w, r2.w);
        if (ragged && q == nvec - 1) {  // keep the row padding at zero
          const int j = 4 * q;
          if (j + 1 >= d) x[s].y = v[s].y = 0.f;
          if (j + 2 >= d) x[s].z = v[s].z = 0.f;
          if (j + 3 >= d) x[s].w = v[s].w = 0.f;
        }
        st_stream(Xr + q, x[s]);
        st_stream(Vr + q, v[s]);
      }
    }
    float acc[Obj::kAcc];
    Obj::init(acc);
    map_row<Obj, VPT>(acc, x, sFirst, nvec, d);
    bool improved;
    const float f = cta_fitness<Obj>(acc, sm, d, pf_old, improved);
    if (improved) {
#pragma unroll
      for (int s = 0; s < VPT; ++s) {
        const int q = threadIdx.x + s * blockDim.x;
        if (q < nvec) st_stream(Pr + q, x[s]);
      }
    }
    if (threadIdx.x == 0) {
      if (improved) {
        a.pf[r] = f;
        ++nimp;
      }
      if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
        const unsigned long long k = pack_key(f, gi);
        best = k < best ? k : best;
      }
    }
  }
  if (cta_finish<Obj>(a, sm, best, nimp)) gbest_epilogue(a, t);
}

// ------------------------------------------------------------ init kernel
// Alg. 1 lines 1-3 (Sec 3.1): x0 = clamp(lo + span U, lo, hi), v0 = -vmax +
// 2 vmax U from the X0 / V0 streams at t = 0; f = F(x0); pf = f (NaN -> +inf);
// PB = x0; every row is a gbest candidate (key_cur = ~0 on entry).
template <class Obj, int VPT>
__global__ void __launch_bounds__(kMaxThreads, (VPT >= 8) ? 1 : 2)
    k_init(const SwarmArgs a) {
  extern __shared__ __align__(16) unsigned char dsmem[];
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float* sFirst = reinterpret_cast<float*>(sG + a.nvec);
  __shared__ RowSmem<Obj> sm;
  const PhiloxKey key{a.seed_lo, a.seed_hi};
  const int nvec = a.nvec, d = a.d;
  const float span = __fsub_rn(a.hi, a.lo);
  const float two_vmax = __fmul_rn(2.f, a.vmax);
  const uint32_t inc_ord = (uint32_t)(a.ctl->key_cur >> 32);
  unsigned long long best = ~0ull;
  for (long long r = blockIdx.x; r < a.n_local; r += gridDim.x) {
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    float4* Xr = reinterpret_cast<float4*>(a.X) + r * nvec;
    float4* Vr = reinterpret_cast<float4*>(a.V) + r * nvec;
    float4* Pr = reinterpret_cast<float4*>(a.PB) + r * nvec;
    float4 x[VPT];
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = threadIdx.x + s * blockDim.x;
      if (q < nvec) {
        const float4 ux = uniforms4(key, kTagX0, 0u, gi, (uint32_t)q);
        const float4 uv = uniforms4(key, kTagV0, 0u, gi, (uint32_t)q);
        float xs[4] = {ux.x, ux.y, ux.z, ux.w};
        float vs[4] = {uv.x, uv.y, uv.z, uv.w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const bool pad = 4 * q + e >= d;
          xs[e] = pad ? 0.f : fminf(fmaxf(__fadd_rn(a.lo, __fmul_rn(span, xs[e])), a.lo), a.hi);
          vs[e] = pad ? 0.f : __fadd_rn(-a.vmax, __fmul_rn(two_vmax, vs[e]));
        }
        x[s] = make_float4(xs[0], xs[1], xs[2], xs[3]);
        st_stream(Xr + q, x[s]);
        st_stream(Vr + q, make_float4(vs[0], vs[1], vs[2], vs[3]));
        st_stream(Pr + q, x[s]);
      }
    }
    float acc[Obj::kAcc];
    Obj::init(acc);
    map_row<Obj, VPT>(acc, x, sFirst, nvec, d);
    bool improved;
    float f = cta_fitness<Obj>(acc, sm, d, 0.f, improved);
    if (threadIdx.x == 0) {
      if (f != f) f = __int_as_float(0x7f800000);  // reading 11: NaN -> +inf
      a.pf[r] = f;
      if (ord_f32(f) < inc_ord) {
        const unsigned long long k = pack_key(f, gi);
        best = k < best ? k : best;
      }
    }
  }
  if (cta_finish<Obj>(a, sm, best, 0)) gbest_epilogue(a, 0u);
  (void)sG;
}

// ---------------------------------------------------------- rebest kernel
// After set_state: pf NaN -> +inf, gbest = lowest index attaining min pf.
__global__ void __launch_bounds__(256) k_rebest(const SwarmArgs a, unsigned t) {
  __shared__ unsigned long long s_best[8];
  __shared__ int s_last;
  unsigned long long best = ~0ull;
  for (long long r = blockIdx.x * (long long)blockDim.x + threadIdx.x; r < a.n_local;
       r += (long long)gridDim.x * blockDim.x) {
    float f = a.pf[r];
    if (f != f) {
      f = __int_as_float(0x7f800000);
      a.pf[r] = f;
    }
    const unsigned long long k = pack_key(f, (uint32_t)(a.row_begin + r));
    best = k < best ? k : best;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    const unsigned long long o = __shfl_xor_sync(kFull, best, off);
    best = o < best ? o : best;
  }
  if ((threadIdx.x & 31) == 0) s_best[threadIdx.x >> 5] = best;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w) best = s_best[w] < best ? s_best[w] : best;
    if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
    __threadfence();
    s_last = (atomicAdd(&a.ctl->done, 1u) == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (s_last) gbest_epilogue(a, t);
}

// ---------------------------------------------------------- select kernel
// world > 1, after ncclAllGather of the records: the global candidate is the
// minimum key over ranks (keys carry global indices, so ties resolve to the
// lowest global index, as one GPU would).  Every rank computes the same bits.
__global__ void __launch_bounds__(128) k_select(const SwarmArgs a) {
  __shared__ unsigned long long s_min;
  __shared__ int s_src;
  const size_t rec = record_bytes(a.nvec * 4);
  if (threadIdx.x < 32) {
    unsigned long long best = ~0ull;
    int src = -1;
    for (int r = threadIdx.x; r < a.world; r += 32) {
      const unsigned long long k =
          *reinterpret_cast<const unsigned long long*>(a.recv + (size_t)r * rec);
      if (k < best) {
        best = k;
        src = r;
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      const unsigned long long o = __shfl_xor_sync(kFull, best, off);
      const int os = __shfl_xor_sync(kFull, src, off);
      if (o < best || (o == best && os >= 0 && (src < 0 || os < src))) {
        best = o;
        src = os;
      }
    }
    if (threadIdx.x == 0) {
      s_min = best;
      s_src = src;
    }
  }
  __syncthreads();
  const unsigned long long cur = a.ctl->key_cur;
  const bool take = s_src >= 0 && s_min < cur;
  if (take) {
    const float4* row = reinterpret_cast<const float4*>(a.recv + (size_t)s_src * rec + 16);
    float4* G4 = reinterpret_cast<float4*>(a.G);
    for (int q = threadIdx.x; q < a.nvec; q += blockDim.x) G4[q] = row[q];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    if (take) a.ctl->key_cur = s_min;
    a.ctl->key_acc = take ? s_min : cur;
  }
}

// ---------------------------------------------------------- debug: objective
template <class Obj, int VPT>
__global__ void __launch_bounds__(kMaxThreads) k_eval(const float* X, long long m, int d,
                                                      int nvec, float* out) {
  extern __shared__ __align__(16) unsigned char dsmem[];
  float* sFirst = reinterpret_cast<float*>(dsmem);
  __shared__ RowSmem<Obj> sm;
  for (long long r = blockIdx.x; r < m; r += gridDim.x) {
    const float4* Xr = reinterpret_cast<const float4*>(X) + r * nvec;
    float4 x[VPT];
#pragma unroll
    for (int s = 0; s < VPT; ++s) {
      const int q = threadIdx.x + s * blockDim.x;
      if (q < nvec) x[s] = Xr[q];
    }
    float acc[Obj::kAcc];
    Obj::init(acc);
    map_row<Obj, VPT>(acc, x, sFirst, nvec, d);
    bool improved;
    const float f = cta_fitness<Obj>(acc, sm, d, 0.f, improved);
    if (threadIdx.x == 0) out[r] = f;
    __syncthreads();
  }
}

// ---------------------------------------------------------- dispatch
constexpr int kVpts[] = {1, 2, 4, 8};

template <class Obj>
struct Kern {
  static const void* step(int vpt) {
    switch (vpt) {
      case 1: return (const void*)k_step<Obj, 1>;
      case 2: return (const void*)k_step<Obj, 2>;
      case 4: return (const void*)k_step<Obj, 4>;
      default: return (const void*)k_step<Obj, 8>;
    }
  }
  static const void* init(int vpt) {
    switch (vpt) {
      case 1: return (const void*)k_init<Obj, 1>;
      case 2: return (const void*)k_init<Obj, 2>;
      case 4: return (const void*)k_init<Obj, 4>;
      default: return (const void*)k_init<Obj, 8>;
    }
  }
  static const void* eval(int vpt) {
    switch (vpt) {
      case 1: return (const void*)k_eval<Obj, 1>;
      case 2: return (const void*)k_eval<Obj, 2>;
      case 4: return (const void*)k_eval<Obj, 4>;
      default: return (const void*)k_eval<Obj, 8>;
    }
  }
  static constexpr bool neighbor = Obj::kNeighbor;
};

enum class Which { Step, Init, Eval };

const void* kernel_for(int objective, Which w, int vpt, bool* neighbor) {
#define PSO_CASE(ID, F)                                                            \
  case ID:                                                                         \
    *neighbor = Kern<F>::neighbor;                                                 \
    return w == Which::Step ? Kern<F>::step(vpt)                                   \
                            : (w == Which::Init ? Kern<F>::init(vpt) : Kern<F>::eval(vpt));
  switch (objective) {
    PSO_ALL_OBJECTIVES(PSO_CASE)
    default:
      return nullptr;
  }
#undef PSO_CASE
}

// CTA shape for a row of nvec float4: the smallest VPT in {1,2,4,8} whose
// thread count fits 256, threads rounded up to a warp multiple.
void shape_for(int nvec, int vpt_override, int* vpt, int* threads) {
  int v = 8;
  for (int c : kVpts) {
    if ((nvec + c - 1) / c <= kMaxThreads) {
      v = c;
      break;
    }
  }
  if (vpt_override == 1 || vpt_override == 2 || vpt_override == 4 || vpt_override == 8) {
    if ((nvec + vpt_override - 1) / vpt_override <= kMaxThreads) v = vpt_override;
  }
  const int t = (nvec + v - 1) / v;
  *vpt = v;
  *threads = ((t + 31) / 32) * 32;
}

size_t dyn_smem(int nvec, bool neighbor, Which w) {
  size_t s = (w == Which::Eval) ? 0 : (size_t)nvec * 16;  // staged G
  if (neighbor) s += (size_t)nvec * 4;                      // first element of each float4
  return s;
}

cudaError_t launch_rows(Which which, int objective, const SwarmArgs& a, const LaunchCfg& c,
                        cudaStream_t s) {
  bool nb = false;
  const void* fn = kernel_for(objective, which, c.vpt, &nb);
  if (!fn) return cudaErrorInvalidDeviceFunction;
  void* args[] = {const_cast<SwarmArgs*>(&a)};
  return cudaLaunchKernel(fn, dim3(c.grid), dim3(c.threads), args, c.smem, s);
}

}  // namespace

bool objective_registered(int objective) {
  bool nb;
  return kernel_for(objective, Which::Step, 1, &nb) != nullptr;
}

cudaError_t plan_launch(int objective, int d, long long n_local, int sm_count, int vpt_override,
                        LaunchCfg* cfg) {
  const int nvec = (d + 3) / 4;
  shape_for(nvec, vpt_override, &cfg->vpt, &cfg->threads);
  bool nb = false;
  const void* fn = kernel_for(objective, Which::Step, cfg->vpt, &nb);
  if (!fn) return cudaErrorInvalidDeviceFunction;
  cfg->smem = dyn_smem(nvec, nb, Which::Step);
  int per_sm = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, cfg->threads, cfg->smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) per_sm = 1;
  cfg->ctas_per_sm = per_sm;
  long long grid = (long long)per_sm * sm_count;
  if (grid > n_local) grid = n_local;
  if (grid < 1) grid = 1;
  cfg->grid = (int)grid;
  return cudaSuccess;
}

cudaError_t launch_step(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s) {
  return launch_rows(Which::Step, objective, a, c, s);
}

cudaError_t launch_init(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s) {
  return launch_rows(Which::Init, objective, a, c, s);
}

cudaError_t launch_rebest(const SwarmArgs& a, unsigned t, cudaStream_t s) {
  long long blocks = (a.n_local + 255) / 256;
  if (blocks > 1024) blocks = 1024;
  if (blocks < 1) blocks = 1;
  k_rebest<<<(unsigned)blocks, 256, 0, s>>>(a, t);
  return cudaGetLastError();
}

cudaError_t launch_select(const SwarmArgs& a, cudaStream_t s) {
  k_select<<<1, 128, 0, s>>>(a);
  return cudaGetLastError();
}

cudaError_t debug_objective(int objective, const float* X_dev, long long m, int d, int pitch,
                            float* out_dev, int sm_count, cudaStream_t s) {
  const int nvec = pitch / 4;
  int vpt, threads;
  shape_for(nvec, 0, &vpt, &threads);
  bool nb = false;
  const void* fn = kernel_for(objective, Which::Eval, vpt, &nb);
  if (!fn) return cudaErrorInvalidDeviceFunction;
  long long grid = m < (long long)sm_count * 4 ? m : (long long)sm_count * 4;
  if (grid < 1) grid = 1;
  void* args[] = {(void*)&X_dev, (void*)&m, (void*)&d, (void*)&nvec, (void*)&out_dev};
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(threads), args, dyn_smem(nvec, nb, Which::Eval),
                          s);
}

}  // namespace fastpso
