// swarm_host.cu — launch planning and dispatch of the fused kernels, and the
// objective-independent kernels (gbest rebest after set_state, multi-GPU select).
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "swarm_kernels.cuh"

namespace fastpso {
namespace {

// ---------------------------------------------------------- rebest kernel
// After set_state: pf NaN -> +inf, gbest = lowest index attaining min pf.
struct NoObj {
  static constexpr int kAcc = 1;
};
__global__ void __launch_bounds__(256) k_rebest(const SwarmArgs a, unsigned t) {
  __shared__ unsigned long long s_best[8];
  __shared__ RowSmem<NoObj> sm;
  const int tid = threadIdx.x, nthr = blockDim.x;
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
  if ((tid & 31) == 0) s_best[tid >> 5] = best;
  __syncthreads();
  if (tid == 0)
    for (int w = 1; w < (nthr >> 5); ++w) best = s_best[w] < best ? s_best[w] : best;
  if (cta_finish<NoObj>(a, sm, tid == 0 ? best : ~0ull, 0, tid, nthr))
    gbest_epilogue<NoObj>(a, sm, t, tid, nthr, ~0ull, -1, a.PB);  // pbest rows given by the host
}

// ---------------------------------------------------------- select kernel
// Exchange mode: fold records for the host.  Synchronous, or at create /
// set_state (into_local): the records of iteration t go into key_cur / G —
// the merge a step kernel's prologue performs, so the next prologue finds
// nothing new (idempotent).  Asynchronous at the end of a pso_step call: the
// records of t - 1 and t are folded into the host's view (key_view / G_view)
// only, leaving the kernels' lagged incumbents untouched, so step(a); step(b)
// is still step(a + b).  Candidates are records strictly better than the
// incumbent (Alg. 1 line 10); the lowest key wins.  Every rank computes the
// same bits.
__global__ void __launch_bounds__(128) k_select(const SwarmArgs a, unsigned t, int into_local) {
  __shared__ unsigned long long s_best;
  __shared__ const float* s_row;
  const bool view_only = a.async_gbest && !into_local;
  if (threadIdx.x == 0) {
    const unsigned long long cur = a.ctl->key_cur;
    unsigned long long best = cur;
    const float* row = nullptr;
    const size_t rec = record_bytes(a.nvec * 4);
    const int n_it = (view_only && t >= a.t_base + 1u) ? 2 : 1;  // records start at t_base
    for (int k = n_it - 1; k >= 0; --k) {
      const unsigned it = t - (unsigned)k;
      if (a.p2p) wait_records(a, it);
      const unsigned char* base = records(a, it);
      for (int r = 0; r < a.xrecs; ++r) {
        const unsigned long long key =
            *reinterpret_cast<const unsigned long long*>(base + (size_t)r * rec);
        if ((key >> 32) < (cur >> 32) && key < best) {
          best = key;
          row = reinterpret_cast<const float*>(base + (size_t)r * rec + 16);
        }
      }
    }
    s_best = best;
    s_row = row;
  }
  __syncthreads();
  const float4* row = reinterpret_cast<const float4*>(s_row);
  float4* dst = reinterpret_cast<float4*>(view_only ? a.G_view : a.G);
  const float4* G4 = reinterpret_cast<const float4*>(a.G);
  for (int q = threadIdx.x; q < a.nvec; q += blockDim.x) {
    const float4 v = row ? row[q] : G4[q];
    dst[q] = v;
    if (!view_only && a.G_view) reinterpret_cast<float4*>(a.G_view)[q] = v;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    if (!view_only) a.ctl->key_cur = s_best;
    a.ctl->key_view = s_best;
  }
}

// ---------------------------------------------------------- empty shard
// A rank that owns no particles (n < world) runs no step kernel, yet its peers
// wait for its record of every iteration.  This one-warp kernel plays the
// rank's part of iteration t.  NVLink exchange: merge the records of t - 1
// into the incumbent (`merge`: what a step kernel's prologue does) and publish
// a "no candidate" record of t to every rank (its epilogue).  NCCL exchange:
// write the "no candidate" record of t into `send` for the all-gather (the host
// folds every iteration's records with k_select).  Records carry the same
// (epoch, iteration) tag as a step kernel's, so switching exchanges is safe.
__global__ void __launch_bounds__(32) k_empty_step(const SwarmArgs a, unsigned t, int merge) {
  const int lane = threadIdx.x;
  const unsigned long long tag = ((unsigned long long)a.epoch << 32) | t;
  if (!a.p2p) {
    if (lane == 0) {
      unsigned long long* hdr = reinterpret_cast<unsigned long long*>(a.send);
      hdr[0] = ~0ull;
      hdr[1] = tag;
      a.ctl->t = t;  // the allreduce exchange's owner kernel reads the slot from it
    }
    return;
  }
  if (merge) {
    int src = -1;
    const unsigned long long best = exchange_merge_warp(a, t - 1u, lane, &src);
    if (src >= 0) {
      const float4* w = reinterpret_cast<const float4*>(merged_gbest_row(a, t - 1u, src));
      for (int q = lane; q < a.nvec; q += 32) {
        const float4 v = w[q];
        reinterpret_cast<float4*>(a.G)[q] = v;
        if (a.G_view) reinterpret_cast<float4*>(a.G_view)[q] = v;
      }
    }
    if (lane == 0) {
      a.ctl->key_cur = best;
      a.ctl->key_view = best;
    }
  }
  if (lane == 0) a.ctl->t = t;
  const size_t rec = record_bytes(a.nvec * 4);
  const size_t off = (size_t)(t & 3u) * a.world * rec + (size_t)a.rank * rec;
  for (int r = lane; r < a.world; r += 32) reinterpret_cast<unsigned long long*>(a.peers[r] + off)[0] = ~0ull;
  __syncwarp();
  for (int r = lane; r < a.world; r += 32) st_release_sys_u64(a.peers[r] + off + 8, tag);
}

// ---------------------------------------------------------- allreduce exchange
// The north star's collective: the records of iteration t are
// reduced into record 0 of slot t & 3 -- ncclAllReduce(min) of the u64 keys,
// then this kernel, then ncclAllReduce(sum) of the row as u32 words.  Here the
// rank whose candidate is the global minimum writes its row, every other rank
// zeros, so the sum is the owner's row bit for bit (a broadcast whose root is
// decided on the device, no host round trip).  Keys hold the global particle
// index, so exactly one rank owns a winning key; with no candidate anywhere
// (key ~0) every rank writes zeros and the merge ignores the record.  The
// iteration comes from the control block (graph-capturable).
__global__ void __launch_bounds__(256) k_owner_row(const SwarmArgs a) {
  const uint32_t t = a.ctl->t;
  unsigned char* rec = const_cast<unsigned char*>(records(a, t));
  const unsigned long long g = *reinterpret_cast<const volatile unsigned long long*>(rec);
  const unsigned long long mine = *reinterpret_cast<const unsigned long long*>(a.send);
  const bool own = g != ~0ull && g == mine;
  const float4* src = reinterpret_cast<const float4*>(a.send + 16);
  float4* dst = reinterpret_cast<float4*>(rec + 16);
  for (int q = threadIdx.x; q < a.nvec; q += blockDim.x)
    dst[q] = own ? src[q] : make_float4(0.f, 0.f, 0.f, 0.f);
  if (threadIdx.x == 0)
    reinterpret_cast<unsigned long long*>(rec)[1] = ((unsigned long long)a.epoch << 32) | t;
}

// ---------------------------------------------------------- NVLink probe
// Proves the peer mappings carry data before the exchange relies on them: a
// system-scope release store of token(rank) into slot `rank` of every rank's
// probe area, then (after the host barrier) acquire loads of our own slots.
__device__ __forceinline__ unsigned long long probe_token(int r) {
  return 0x50534F5000000000ull | (unsigned)(r + 1);
}
__global__ void __launch_bounds__(32) k_p2p_probe(const SwarmArgs a, int phase, int* ok) {
  const int lane = threadIdx.x;
  if (phase == 0) {
    for (int r = lane; r < a.world; r += 32)
      st_release_sys_u64(a.peers[r] + a.probe_off + 8ull * a.rank, probe_token(a.rank));
    return;
  }
  unsigned char* mine = const_cast<unsigned char*>(a.recv) + a.probe_off;
  int good = 1;
  for (int r = lane; r < a.world; r += 32) {
    good &= ld_acquire_sys_u64(mine + 8ull * r) == probe_token(r);
    reinterpret_cast<unsigned long long*>(mine)[r] = 0ull;
  }
  good = __all_sync(kFull, good);
  if (lane == 0) *ok = good;
}

// ---------------------------------------------------------- materialize PB
// Restores the plain layout (X holds x, PB holds pb, pbx = 0) before the host
// reads whole matrices.  pbx bit 0: lazy pbest row (PB == x, not stored);
// bit 1 (column split only): x lives in the PB array, a non-lazy pbest in the
// X array (swarm_colsplit.cuh).  One warp per flagged row.
__global__ void __launch_bounds__(256) k_materialize_pb(const SwarmArgs a) {
  const int lane = threadIdx.x & 31;
  const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long r = blockIdx.x * (long long)(blockDim.x >> 5) + (threadIdx.x >> 5); r < a.n_local;
       r += warps) {
    const int fl = a.pbx[r];
    if (!fl) continue;
    float4* x = reinterpret_cast<float4*>(a.X) + r * a.nvec;
    float4* pb = reinterpret_cast<float4*>(a.PB) + r * a.nvec;
    for (int q = lane; q < a.nvec; q += 32) {
      if (fl == 1) {
        pb[q] = x[q];
      } else if (fl == 3) {
        x[q] = pb[q];
      } else {  // 2: swap the slots
        const float4 t = x[q];
        x[q] = pb[q];
        pb[q] = t;
      }
    }
    __syncwarp();
    if (lane == 0) a.pbx[r] = 0;
  }
}

// ---------------------------------------------------------- dispatch
enum class Which { StepReg, StepTma, Init, Eval, GridRes };

int vpt_index(int vpt) { return vpt == 1 ? 0 : vpt == 2 ? 1 : vpt == 4 ? 2 : 3; }

const void* kernel_for(int objective, Which w, int vpt, bool bounds, bool* neighbor) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return nullptr;
  *neighbor = t->neighbor;
  const int i = vpt_index(vpt), b = bounds ? 1 : 0;
  switch (w) {
    case Which::StepReg: return t->step_reg[i][b];
    case Which::StepTma: return t->step_tma[i][b];
    case Which::GridRes: return t->gridres[i][b];
    case Which::Init: return t->init[i];
    default: return t->eval[i];
  }
}

// CTA shape for a row of nvec float4: the smallest VPT in {1,2,4,8} whose
// thread count fits 256, threads rounded up to a warp multiple.
void shape_for(int nvec, int vpt_override, int* vpt, int* threads, int max_threads = kMaxThreads) {
  static const int kVpts[] = {1, 2, 4, 8};
  int v = 8;
  for (int c : kVpts) {
    if ((nvec + c - 1) / c <= max_threads) {
      v = c;
      break;
    }
  }
  if (vpt_override == 1 || vpt_override == 2 || vpt_override == 4 || vpt_override == 8) {
    if ((nvec + vpt_override - 1) / vpt_override <= max_threads) v = vpt_override;
  }
  const int t = (nvec + v - 1) / v;
  *vpt = v;
  *threads = ((t + 31) / 32) * 32;
}

constexpr size_t kSmemPerSm = 228 * 1024;       // B200 unified L1/shared per SM
constexpr size_t kSmemPerCtaMax = 227 * 1024;   // opt-in maximum per CTA
constexpr size_t kStaticReserve = 4096;         // static shared (<= 3 KB) + per-CTA reservation
// persistent streaming kernel: used automatically up to this many rows per CTA.
// 0 = opt-in only (PSO_PERSIST=1): measured faster where most rows are lazy
// (Griewank 10000 x 2000: 66.1 -> 56.6 us per iteration) but slower on C3
// (Rosenbrock 10000 x 1000: 34.4 -> 37.3 us) and NS_R8 (75.9 -> 80.3 us), and
// the lazy share is not known when the plan is made.
constexpr long long kPersistMaxRowsPerCta = 0;
constexpr long long kResidentElems = 8192;      // resident path: n d <= this

}  // namespace

// cudaFuncAttributeMaxDynamicSharedMemorySize is one setting per kernel function
// (per device), shared by every handle of the process: it is only ever RAISED,
// to the largest ring any handle planned, so creating a handle never lowers the
// limit an older handle of the same instantiation launches with.
cudaError_t allow_dynamic_smem(const void* fn, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<int, const void*>, size_t> granted;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lock(mu);
  size_t& g = granted[{dev, fn}];
  if (bytes <= g) return cudaSuccess;
  e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) g = bytes;
  return e;
}

bool objective_registered(int objective) {
  bool nb;
  return kernel_for(objective, Which::Init, 1, false, &nb) != nullptr;
}

namespace {

// Ring depth for stages of `stage_bytes` next to `fixed` bytes, at `ctas` CTAs per SM.
int ring_stages(size_t fixed, size_t stage_bytes, int ctas) {
  size_t budget = kSmemPerSm / ctas - kStaticReserve;
  if (budget > kSmemPerCtaMax - kStaticReserve) budget = kSmemPerCtaMax - kStaticReserve;
  return budget > fixed ? (int)((budget - fixed) / stage_bytes) : 0;
}

// One cluster shape: C CTAs per row, the ring sized for one CTA per SM.  Fills
// *cfg and reports how many SMs its clusters cover (0 if it does not fit).
cudaError_t cluster_shape(const KernelTable* t, int nvec, int C, const PlanHints& h, LaunchCfg* cfg,
                          int* sms_covered) {
  *sms_covered = 0;
  const int chunk = (nvec + C - 1) / C;
  if (C < 2 || C > 16 || chunk > 2048) return cudaSuccess;
  int vpt, compute;
  shape_for(chunk, h.vpt, &vpt, &compute, kMaxThreadsCluster);
  if ((chunk + vpt - 1) / vpt > kMaxThreadsCluster) return cudaSuccess;
  const void* fn = t->step_cluster[vpt_index(vpt)][h.bounds ? 1 : 0];
  const size_t crow = (size_t)chunk * 16, btab = h.bounds ? 4 * crow : 0;
  const int per_sm = (h.ctas >= 1 && h.ctas <= 4) ? h.ctas : 1;  // CTAs per SM to size the ring for
  cudaError_t e;
  int stages = ring_stages(crow + btab, 3 * crow, per_sm);
  if (per_sm == 1) {  // one CTA per SM: the exact budget next to the kernel's static shared memory
    cudaFuncAttributes fa{};
    if ((e = cudaFuncGetAttributes(&fa, fn)) != cudaSuccess) return e;
    const size_t budget = kSmemPerCtaMax - fa.sharedSizeBytes, fixed = crow + btab;
    stages = budget > fixed ? (int)((budget - fixed) / (3 * crow)) : 0;
  }
  if (h.stages >= 2 && h.stages < stages) stages = h.stages;
  if (stages > kClusterStages) stages = kClusterStages;
  if (stages < 2) return cudaSuccess;
  const size_t smem = crow + btab + (size_t)stages * 3 * crow;
  if (C > 8 &&
      (e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1)) != cudaSuccess)
    return e;
  if ((e = allow_dynamic_smem(fn, smem)) != cudaSuccess) return e;
  cudaLaunchConfig_t lc{};
  lc.gridDim = dim3(C);
  lc.blockDim = dim3(compute + 64);
  lc.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = C;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  lc.attrs = attr;
  lc.numAttrs = 1;
  int ncl = 0;
  if ((e = cudaOccupancyMaxActiveClusters(&ncl, fn, &lc)) != cudaSuccess) {
    cudaGetLastError();  // e.g. a cluster size the device cannot co-schedule
    return cudaSuccess;
  }
  if (ncl < 1) return cudaSuccess;
  cfg->cluster = C;
  cfg->chunk = chunk;
  cfg->vpt = vpt;
  cfg->compute = compute;
  cfg->threads = compute + 64;
  cfg->tma = 1;
  cfg->stages = stages;
  cfg->smem = smem;
  cfg->grid = ncl * C;  // clipped to the rows by the caller
  cfg->ctas_per_sm = 1;
  *sms_covered = ncl * C / per_sm;
  return cudaSuccess;
}

// Cluster path (NEXT-3): rows of more than 2048 float4 (d > 8192), or forced
// (PSO_CLUSTER = any size 2-16).  Automatic size: the smallest power of two
// whose column block is <= 1024 float4 (d only, never n or the world size, so
// the block combine order -- and every fitness bit -- is the same on every
// rank).  Measured at W16K (Griewank 16384 x 16384, round 2): C = 4 (132 SMs,
// 4 stages) 821 us; C = 3 (135 SMs, 3 stages) 1122; C = 5 (130 SMs) 978; C = 8
// 1478; C = 16 (2 CTAs per SM) 1626 -- covering more SMs does not pay: the
// cluster's per-row handshake, not SM coverage, set the pace.
cudaError_t plan_cluster(const KernelTable* t, int nvec, long long n_local, const PlanHints& h,
                         LaunchCfg* cfg) {
  int C = h.cluster;
  if (C <= 0) {
    C = 2;
    while (C < 16 && (nvec + C - 1) / C > 1024) C *= 2;
  }
  int sms = 0;
  LaunchCfg c = *cfg;
  cudaError_t e = cluster_shape(t, nvec, C, h, &c, &sms);
  if (e != cudaSuccess) return e;
  if (sms == 0) return cudaErrorInvalidConfiguration;
  *cfg = c;
  const long long clusters = std::min<long long>(cfg->grid / cfg->cluster, n_local);
  cfg->grid = (int)(clusters * cfg->cluster);
  return cudaSuccess;
}

}  // namespace

cudaError_t plan_launch(int objective, int d, long long n_local, int sm_count, const PlanHints& h,
                        LaunchCfg* cfg) {
  const KernelTable* tab = kernel_table(objective);
  if (!tab) return cudaErrorInvalidDeviceFunction;
  const bool nb = tab->neighbor;
  const int nvec = (d + 3) / 4;
  const size_t row = (size_t)nvec * 16;
  const size_t btab = h.bounds ? 4 * row : 0;  // per-dimension bounds table in shared memory
  const size_t first = nb ? (size_t)nvec * 4 : 0;
  cfg->bounds = h.bounds ? 1 : 0;
  cfg->init_smem = 0;
  cfg->resident = cfg->gridres = cfg->cluster = cfg->persist = 0;
  cudaError_t e;

  // init kernel: one CTA per row, looping over the row's float4s
  {
    int iv, it;
    shape_for(nvec <= 2048 ? nvec : 2048, 0, &iv, &it);
    cfg->init_vpt = iv;
    cfg->init_threads = it;
  }

  // ---- wide rows: thread-block cluster per row
  if (nvec > 2048 || h.cluster > 0) return plan_cluster(tab, nvec, n_local, h, cfg);
  shape_for(nvec, h.vpt, &cfg->vpt, &cfg->compute);
  int vi = vpt_index(cfg->vpt);
  const int bi = h.bounds ? 1 : 0;

  // ---- resident single-CTA path for tiny swarms (single GPU only)
  if (h.allow_resident && nvec <= 32 && n_local * nvec * 4 <= kResidentElems) {
    const size_t smem =
        (size_t)n_local * nvec * 16 * 3 + (size_t)nvec * 16 + btab + (size_t)n_local * 4;
    const void* fn = tab->resident[bi];
    if (smem <= kSmemPerCtaMax - kStaticReserve &&
        allow_dynamic_smem(fn, smem) ==
            cudaSuccess) {
      int gs = 1;
      while (gs < nvec) gs <<= 1;
      const long long rpw = 32 / gs;
      long long warps = (n_local + rpw - 1) / rpw;
      if (warps > 32) warps = 32;
      cfg->resident = 1;
      cfg->resident_threads = 32 * (int)(warps < 1 ? 1 : warps);
      cfg->resident_smem = smem;
    }
    cudaGetLastError();
  }

  // ---- streaming kernels: TMA pipeline for rows of >= 256 dims unless forced.
  // Shape: (float4 per thread, CTAs per SM) from d only (never from n, so the
  // per-row reduction order -- and every fitness bit -- is the same for every
  // swarm size and world size).  Rule (measured, profiles/r01_tune_*): reach
  // 16 compute warps per SM with >= 3 ring stages per CTA, and among shapes
  // that do, prefer 2 float4 per thread (the per-row, per-warp bookkeeping --
  // barrier waits, partial combine, arrivals -- is amortised over 8 elements
  // per lane instead of 4; C3 Rosenbrock 10k x 1000: 45.8 -> 41.6 us).
  bool tma = h.kernel == 1 || (h.kernel == -1 && nvec >= 64);
  if (tma) {
    // (float4 per thread, max compute threads) in order of preference; the
    // 512-thread (wide) instantiations exist for VPT 2 and 4
    static const int kPref[][2] = {{2, 256}, {1, 256}, {2, 512}, {4, 256}, {4, 512}, {8, 256}};
    const int cap = (h.ctas >= 1 && h.ctas <= 8) ? h.ctas : 8;
    int best_v = 0, best_c = 0, best_stages = 0, best_threads = 0, best_score = -1, best_wide = 0;
    for (const auto& pr : kPref) {
      const int v = pr[0], maxt = pr[1];
      if (h.vpt && v != h.vpt) continue;
      const int t = (nvec + v - 1) / v;
      if (t > maxt && v != 8) continue;
      if (maxt > kMaxThreads && t <= kMaxThreads) continue;  // the narrow variant covers it
      const int compute = ((t < maxt ? t : maxt) + 31) / 32 * 32;
      const void* fn = maxt > kMaxThreads ? tab->step_tma_w[vpt_index(v)][bi]
                                          : tab->step_tma[vpt_index(v)][bi];
      int by_regs = 0;
      if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&by_regs, fn, compute + 64, 0)) !=
          cudaSuccess)
        return e;
      int hi = by_regs < cap ? by_regs : cap;
      // fewest CTAs that reach 16 compute warps, else as many as fit
      const int want = (16 * 32 + compute - 1) / compute;
      if (hi > want) hi = want;
      int c = hi;
      for (; c >= 1; --c)
        if (ring_stages(row + btab, 3 * row, c) >= 3) break;
      if (c < 1)  // two rows in flight only if nothing else fits
        for (c = hi; c >= 1 && ring_stages(row + btab, 3 * row, c) < 2; --c) {
        }
      if (c < 1) continue;
      const int warps = c * compute / 32;
      const int score = warps < 16 ? warps : 16;
      if (score > best_score) {
        best_score = score;
        best_v = v;
        best_c = c;
        best_threads = compute;
        best_stages = ring_stages(row + btab, 3 * row, c);
        best_wide = maxt > kMaxThreads ? 1 : 0;
      }
    }
    tma = false;
    if (best_score > 0) {
      cfg->vpt = best_v;
      cfg->compute = best_threads;
      vi = vpt_index(best_v);
      int stages = best_stages;
      if (h.stages >= 2 && h.stages <= kMaxStages) stages = stages < h.stages ? stages : h.stages;
      if (stages > kMaxStages) stages = kMaxStages;
      const void* fn = best_wide ? tab->step_tma_w[vi][bi] : tab->step_tma[vi][bi];
      const int threads = cfg->compute + 64;  // + producer warp + finaliser warp
      if (stages >= 2) {
        const size_t smem = row + btab + (size_t)stages * 3 * row;
        if ((e = allow_dynamic_smem(fn, smem)) !=
            cudaSuccess)
          return e;
        int per_sm = 0;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem)) !=
            cudaSuccess)
          return e;
        if (per_sm >= 1) {
          tma = true;
          cfg->tma = 1;
          cfg->wide = best_wide;
          cfg->stages = stages;
          cfg->threads = threads;
          cfg->smem = smem;
          cfg->ctas_per_sm = per_sm < best_c ? per_sm : best_c;
        }
      }
    }
    if (!tma) shape_for(nvec, h.vpt, &cfg->vpt, &cfg->compute), vi = vpt_index(cfg->vpt);
  }
  if (!tma) {
    const void* fn = tab->step_reg[vi][bi];
    cfg->tma = 0;
    cfg->wide = 0;
    cfg->stages = 0;
    cfg->threads = cfg->compute;
    cfg->smem = row + btab + first;
    if ((e = allow_dynamic_smem(fn, cfg->smem)) != cudaSuccess)
      return e;
    int per_sm = 0;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, cfg->threads, cfg->smem)) !=
        cudaSuccess)
      return e;
    cfg->ctas_per_sm = per_sm < 1 ? 1 : per_sm;
  }
  long long grid = (long long)cfg->ctas_per_sm * sm_count;
  if (grid > n_local) grid = n_local;
  if (grid < 1) grid = 1;
  cfg->grid = (int)grid;

  // ---- grid-resident path: the whole swarm in the grid's shared memory
  if (h.allow_resident && !cfg->resident && cfg->tma && nvec >= 64 && h.persist != 1) {
    const void* fn = tab->gridres[vi][bi];
    for (int per = cfg->ctas_per_sm; per >= 1 && !cfg->gridres; --per) {
      long long g = (long long)per * sm_count;
      if (g > n_local) g = n_local;
      const long long rows = (n_local + g - 1) / g;
      const size_t smem = row + btab + (size_t)rows * 3 * row + (size_t)rows * 4;
      if (smem > kSmemPerCtaMax - kStaticReserve || smem * per > kSmemPerSm - per * kStaticReserve)
        continue;
      if (allow_dynamic_smem(fn, smem) !=
          cudaSuccess) {
        cudaGetLastError();
        continue;
      }
      int occ = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, cfg->compute, smem) != cudaSuccess) {
        cudaGetLastError();
        continue;
      }
      if ((long long)occ * sm_count < g) continue;  // cooperative: every CTA co-resident
      cfg->gridres = 1;
      cfg->gridres_grid = (int)g;
      cfg->gridres_rows = (int)rows;
      cfg->gridres_smem = smem;
    }
  }

  // ---- persistent streaming kernel (swarm_persist.cuh): the narrow TMA shape,
  // a whole pso_step call per cooperative launch, for swarms whose rows per CTA
  // are few enough that the per-iteration kernel boundary shows (PSO_PERSIST=1
  // forces it, 0 disables it)
  if (h.allow_resident && !cfg->resident && !cfg->gridres && cfg->tma && !cfg->wide && h.persist != 0) {
    const long long rows_per_cta = (n_local + cfg->grid - 1) / cfg->grid;
    if (h.persist == 1 || rows_per_cta <= kPersistMaxRowsPerCta) {
      const void* fn = tab->persist[vi][bi];
      if ((e = allow_dynamic_smem(fn, cfg->smem)) != cudaSuccess) return e;
      int occ = 0;
      if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, cfg->threads, cfg->smem)) !=
          cudaSuccess)
        return e;
      const int per = occ < cfg->ctas_per_sm ? occ : cfg->ctas_per_sm;
      long long g = (long long)per * sm_count;
      if (g > n_local) g = n_local;
      if (per >= 1 && g >= 1) {
        cfg->persist = 1;
        cfg->persist_grid = (int)g;
      }
    }
  }
  return cudaSuccess;
}

cudaError_t launch_step(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  const int vi = vpt_index(c.vpt), bi = c.bounds ? 1 : 0;
  int stages = c.stages;
  int C = c.cluster, chunk = c.chunk;
  void* args[] = {const_cast<SwarmArgs*>(&a), &stages, &C, &chunk};
  cudaLaunchConfig_t lc{};
  lc.gridDim = dim3(c.grid);
  lc.blockDim = dim3(c.threads);
  lc.dynamicSmemBytes = c.smem;
  lc.stream = s;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (c.pdl) {  // overlap this grid's launch with the previous step kernel's drain
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  const void* fn;
  if (c.cluster) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = C;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
    fn = t->step_cluster[vi][bi];
  } else {
    fn = !c.tma ? t->step_reg[vi][bi] : c.wide ? t->step_tma_w[vi][bi] : t->step_tma[vi][bi];
  }
  lc.attrs = attr;
  lc.numAttrs = na;
  return cudaLaunchKernelExC(&lc, fn, args);
}

cudaError_t launch_resident(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                            cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  void* args[] = {const_cast<SwarmArgs*>(&a), &iters};
  return cudaLaunchKernel(t->resident[c.bounds ? 1 : 0], dim3(1), dim3(c.resident_threads), args,
                          c.resident_smem, s);
}

cudaError_t launch_gridres(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                           cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  void* args[] = {const_cast<SwarmArgs*>(&a), &iters};
  return cudaLaunchCooperativeKernel(t->gridres[vpt_index(c.vpt)][c.bounds ? 1 : 0],
                                     dim3(c.gridres_grid), dim3(c.compute), args, c.gridres_smem, s);
}

cudaError_t launch_persist(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                           cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  int stages = c.stages;
  void* args[] = {const_cast<SwarmArgs*>(&a), &iters, &stages};
  return cudaLaunchCooperativeKernel(t->persist[vpt_index(c.vpt)][c.bounds ? 1 : 0],
                                     dim3(c.persist_grid), dim3(c.threads), args, c.smem, s);
}

cudaError_t launch_init(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  long long grid = a.n_local < 4LL * 148 * 2 ? a.n_local : 4LL * 148 * 2;
  if (grid < 1) grid = 1;
  void* args[] = {const_cast<SwarmArgs*>(&a)};
  return cudaLaunchKernel(t->init[vpt_index(c.init_vpt)], dim3((unsigned)grid),
                          dim3(c.init_threads), args, 0, s);
}

// ---------------------------------------------------------- column split
// A launch with programmatic stream serialization (PDL) when `pdl`: the kernel
// is scheduled while the previous one drains and waits for it with
// griddepcontrol.wait before its first global read.
cudaError_t launch_pdl(const void* fn, dim3 grid, dim3 block, void** args, size_t smem, cudaStream_t s,
                       int pdl) {
  cudaLaunchConfig_t lc{};
  lc.gridDim = grid;
  lc.blockDim = block;
  lc.dynamicSmemBytes = smem;
  lc.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  lc.attrs = attr;
  lc.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelExC(&lc, fn, args);
}

cudaError_t plan_colsplit(int objective, int tile, int tiles_local, long long n, int sm_count,
                          bool bounds, LaunchCfg* cfg) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  if (tile < 1 || tiles_local < 1 || n < 1) return cudaErrorInvalidConfiguration;
  // k_col_step's shared memory: a G cache of 2 slots x {g [, 4 bounds tiles]},
  // then the ring of {x, v, pb} stages
  const size_t stage = (size_t)3 * tile * 16, gcache = (size_t)2 * (bounds ? 5 : 1) * tile * 16;
  int ctas = bounds ? 1 : 2;  // ~100 registers x 320 threads: 2 CTAs per SM
  if (const char* v = std::getenv("PSO_COL_CTAS")) ctas = std::max(1, std::min(2, std::atoi(v)));
  const void* fn = t->col_step[bounds ? 1 : 0];
  // the exact budget: the SM's shared memory over its CTAs, less the per-CTA
  // reservation and the kernel's static shared memory (512-float4 tiles: 16 KB
  // of cache + 4 stages of 24 KB fit two CTAs with 128 B to spare)
  cudaFuncAttributes fa{};
  cudaError_t e = cudaFuncGetAttributes(&fa, fn);
  if (e != cudaSuccess) return e;
  int dev = 0, per_sm = 0, reserved = 0, optin = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev)) != cudaSuccess ||
      (e = cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev)) != cudaSuccess ||
      (e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev)) != cudaSuccess)
    return e;
  long long budget = (long long)per_sm / ctas - reserved - (long long)fa.sharedSizeBytes;
  budget = std::min(budget, (long long)optin - (long long)fa.sharedSizeBytes);
  int stages = budget > (long long)gcache ? (int)((budget - (long long)gcache) / (long long)stage) : 0;
  int max_st = 4;  // 4 tiles in flight per CTA cover the HBM latency
  if (const char* v = std::getenv("PSO_COL_STAGES")) max_st = std::max(2, std::min(kMaxStages, std::atoi(v)));
  if (stages > max_st) stages = max_st;
  if (stages < 2) return cudaErrorInvalidConfiguration;
  const size_t smem = gcache + (size_t)stages * stage;
  e = allow_dynamic_smem(fn, smem);
  if (e != cudaSuccess) return e;
  const long long items = n * tiles_local;
  long long grid = (long long)sm_count * ctas;
  if (grid > items) grid = items;
  cfg->colsplit = 1;
  cfg->chunk = tile;
  cfg->col_grid = (int)grid;
  cfg->col_stages = stages;
  cfg->col_smem = smem;
  cfg->threads = kColCompute + 64;
  cfg->compute = kColCompute;
  cfg->grid = (int)grid;
  cfg->ctas_per_sm = ctas;
  cfg->tma = 1;
  cfg->stages = stages;
  cfg->smem = smem;
  cfg->bounds = bounds ? 1 : 0;
  const int rows_per_cta = kColDecideThreads / 32;  // one warp per row
  long long dg = (n + rows_per_cta - 1) / rows_per_cta;
  if (dg > (long long)sm_count * 4) dg = (long long)sm_count * 4;
  cfg->col_decide_grid = (int)(dg < 1 ? 1 : dg);
  return cudaSuccess;
}

cudaError_t launch_col_step(int objective, const SwarmArgs& a, const LaunchCfg& c, int init,
                            cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  int stages = c.col_stages;
  void* args[] = {const_cast<SwarmArgs*>(&a), &init, &stages};
  return launch_pdl(t->col_step[c.bounds ? 1 : 0], dim3(c.col_grid), dim3(c.threads), args,
                    c.col_smem, s, c.pdl);
}

cudaError_t launch_col_decide(int objective, const SwarmArgs& a, const LaunchCfg& c, int init,
                              cudaStream_t s) {
  const KernelTable* t = kernel_table(objective);
  if (!t) return cudaErrorInvalidDeviceFunction;
  void* args[] = {const_cast<SwarmArgs*>(&a), &init};
  return launch_pdl(t->col_decide, dim3(c.col_decide_grid), dim3(kColDecideThreads), args, 0, s, c.pdl);
}

cudaError_t launch_rebest(const SwarmArgs& a, unsigned t, cudaStream_t s) {
  long long blocks = (a.n_local + 255) / 256;
  if (blocks > 1024) blocks = 1024;
  if (blocks < 1) blocks = 1;
  k_rebest<<<(unsigned)blocks, 256, 0, s>>>(a, t);
  return cudaGetLastError();
}

cudaError_t launch_materialize_pb(const SwarmArgs& a, cudaStream_t s) {
  if (!a.lazy_pb || a.n_local < 1) return cudaSuccess;
  long long blocks = (a.n_local + 7) / 8;
  if (blocks > 2048) blocks = 2048;
  k_materialize_pb<<<(unsigned)blocks, 256, 0, s>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_owner_row(const SwarmArgs& a, cudaStream_t s) {
  k_owner_row<<<1, 256, 0, s>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_p2p_probe(const SwarmArgs& a, int phase, int* ok_dev, cudaStream_t s) {
  k_p2p_probe<<<1, 32, 0, s>>>(a, phase, ok_dev);
  return cudaGetLastError();
}

cudaError_t launch_empty_step(const SwarmArgs& a, unsigned t, bool merge, cudaStream_t s) {
  k_empty_step<<<1, 32, 0, s>>>(a, t, merge ? 1 : 0);
  return cudaGetLastError();
}

cudaError_t launch_select(const SwarmArgs& a, unsigned t, bool into_local, cudaStream_t s) {
  k_select<<<1, 128, 0, s>>>(a, t, into_local ? 1 : 0);
  return cudaGetLastError();
}

cudaError_t debug_objective(int objective, const float* X_dev, long long m, int d, int pitch,
                            float* out_dev, int sm_count, cudaStream_t s) {
  const int nvec = pitch / 4;
  int vpt, threads;
  shape_for(nvec <= 2048 ? nvec : 2048, 0, &vpt, &threads);
  bool nb = false;
  const void* fn = kernel_for(objective, Which::Eval, vpt, false, &nb);
  if (!fn) return cudaErrorInvalidDeviceFunction;
  long long grid = m < (long long)sm_count * 4 ? m : (long long)sm_count * 4;
  if (grid < 1) grid = 1;
  void* args[] = {(void*)&X_dev, (void*)&m, (void*)&d, (void*)&nvec, (void*)&out_dev};
  return cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(threads), args, 0, s);
}

}  // namespace fastpso

