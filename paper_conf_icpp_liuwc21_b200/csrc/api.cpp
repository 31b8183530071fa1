// api.cpp — the C ABI of include/fastpso.h: validation, the per-handle device
// arena (the paper's GPU memory caching: one allocation reused for the
// whole run), the iteration loop of Alg. 1 as kernel launches,
// the synchronous particle-split gbest exchange over NCCL, state I/O,
// counters and error handling.
#include "fastpso.h"

#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <string>
#include <utility>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "kernels.h"

using namespace fastpso;

namespace {

// NVTX ranges around every entry point that enqueues or waits for GPU work
// (header-only NVTX v3: free unless a profiler such as nsys / ncu attaches).
nvtxDomainHandle_t nvtx_domain() {
  static nvtxDomainHandle_t d = nvtxDomainCreateA("fastpso");
  return d;
}
struct NvtxRange {
  explicit NvtxRange(const char* name) {
    nvtxEventAttributes_t ev{};
    ev.version = NVTX_VERSION;
    ev.size = NVTX_EVENT_ATTRIB_STRUCT_SIZE;
    ev.messageType = NVTX_MESSAGE_TYPE_ASCII;
    ev.message.ascii = name;
    nvtxDomainRangePushEx(nvtx_domain(), &ev);
  }
  ~NvtxRange() { nvtxDomainRangePop(nvtx_domain()); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

thread_local std::string g_last_error;

pso_status fail(pso_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return s;
}

// ------------------------------------------------------------ NCCL (dlopen)
// Minimal ABI subset of nccl.h (stable across NCCL 2.x).
typedef struct ncclComm* ncclComm_t;
typedef struct {
  char internal[128];
} ncclUniqueId;
typedef int ncclResult_t;  // ncclSuccess == 0
enum { kNcclUint8 = 1, kNcclUint32 = 3, kNcclUint64 = 5 };  // ncclDataType_t
enum { kNcclSum = 0, kNcclMin = 3 };                          // ncclRedOp_t

struct NcclApi {
  void* handle = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommCount)(ncclComm_t, int*) = nullptr;
  ncclResult_t (*CommUserRank)(ncclComm_t, int*) = nullptr;
  ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  std::string error;
};

NcclApi* nccl() {
  static NcclApi api;
  static bool tried = false;
  if (tried) return api.handle ? &api : nullptr;
  tried = true;
  const char* env = std::getenv("PSO_NCCL_LIB");
  const char* names[] = {env, "libnccl.so.2", "libnccl.so"};
  for (const char* n : names) {
    if (!n || !*n) continue;
    // Prefer an NCCL already loaded into the process (e.g. by PyTorch).
    api.handle = dlopen(n, RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
    if (!api.handle) api.handle = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
    if (api.handle) break;
  }
  if (!api.handle) {
    const char* e = dlerror();
    api.error = e ? e : "libnccl.so.2 not found";
    return nullptr;
  }
#define PSO_SYM(field, name)                                       \
  *(void**)(&api.field) = dlsym(api.handle, name);                 \
  if (!api.field) {                                                \
    api.error = std::string("missing NCCL symbol ") + name;        \
    api.handle = nullptr;                                          \
    return nullptr;                                                \
  }
  PSO_SYM(GetUniqueId, "ncclGetUniqueId")
  PSO_SYM(CommInitRank, "ncclCommInitRank")
  PSO_SYM(CommDestroy, "ncclCommDestroy")
  PSO_SYM(CommCount, "ncclCommCount")
  PSO_SYM(CommUserRank, "ncclCommUserRank")
  PSO_SYM(CommGetAsyncError, "ncclCommGetAsyncError")
  PSO_SYM(AllGather, "ncclAllGather")
  PSO_SYM(AllReduce, "ncclAllReduce")
  PSO_SYM(GetErrorString, "ncclGetErrorString")
#undef PSO_SYM
  return &api;
}

const char* nccl_str(ncclResult_t r) {
  NcclApi* a = nccl();
  return (a && a->GetErrorString) ? a->GetErrorString(r) : "nccl error";
}

// ------------------------------------------------------------ the handle
size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

}  // namespace

struct pso_swarm {
  // problem
  int64_t n = 0, n_local = 0, row_begin = 0;
  int32_t d = 0, pitch = 0, objective = 0;
  float w = 0, c1 = 0, c2 = 0, lo = 0, hi = 0, vmax = 1;
  uint64_t seed = 0;
  // placement
  int device = 0, sm_count = 0, rank = 0, world = 1;
  bool xchg = false;  // run the all-gather + select exchange (world > 1, or forced for testing)
  // column split (NEXT-3): all n rows, columns [col_begin, col_begin + d_local)
  bool colsplit = false;
  int32_t col_begin = 0, d_local = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  ncclComm_t comm = nullptr;
  uint32_t flags = 0;
  // memory
  void* arena = nullptr;
  size_t arena_bytes = 0;
  SwarmArgs args{};
  LaunchCfg cfg{};
  // run state
  uint64_t t = 0;
  bool poisoned = false;
  uint64_t launches = 0;
  struct Timed {
    cudaEvent_t start, stop;
    uint64_t steps;  // step kernels (iterations) between the two events
  };
  std::vector<Timed> events;
  size_t events_used = 0;
  double timed_ms = 0;
  uint64_t timed_count = 0;
  bool inited = false;  // pso_init done (or state set)
  // NVLink peer exchange (pso_p2p_connect)
  std::vector<void*> ipc_opened;
  void* peers_dev = nullptr;
  // NCCL exchange: captured [step, all-gather] x kGraphIters, one per slot phase
  cudaGraphExec_t nccl_graph[4] = {nullptr, nullptr, nullptr, nullptr};
  bool graph_off = false;
  bool allreduce = false;  // PSO_FLAG_ALLREDUCE: NCCL exchange as allreduce-min + sum-broadcast
};

namespace {

constexpr int kGraphIters = 4;  // iterations per captured NCCL-exchange graph

pso_status cuda_fail(pso_swarm* h, cudaError_t e, const char* what) {
  if (h) h->poisoned = true;
  cudaGetLastError();  // clear a sticky launch error where possible
  return fail(PSO_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
}

#define PSO_CUDA(h, call)                                      \
  do {                                                         \
    cudaError_t _e = (call);                                   \
    if (_e != cudaSuccess) return cuda_fail((h), _e, #call);   \
  } while (0)

pso_status check_handle(pso_swarm* h) {
  if (!h) return fail(PSO_ERR_INVALID, "NULL handle");
  if (h->poisoned) return fail(PSO_ERR_POISONED, "handle poisoned by an earlier CUDA/NCCL error");
  return PSO_OK;
}

// Calls that read or advance the swarm need it initialised (pso_init / set_state).
pso_status check_ready(pso_swarm* h) {
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (!h->inited) return fail(PSO_ERR_INVALID, "swarm not initialised: call pso_init (deferred init)");
  return PSO_OK;
}

// Make the handle's device current for this call.
pso_status use_device(pso_swarm* h) {
  PSO_CUDA(h, cudaSetDevice(h->device));
  return PSO_OK;
}

// The NCCL exchange of one iteration (records of iteration t into slot t & 3):
// the all-gather of every rank's record, or -- PSO_FLAG_ALLREDUCE, the north
// star's collective -- an allreduce-min of the u64 keys into record 0, the
// owner kernel (the winner's row or zeros), and an allreduce-sum of the row as
// u32 words (a bit-exact broadcast from the device-decided owner).
ncclResult_t nccl_exchange(pso_swarm* h, NcclApi* a, uint64_t t, bool* launched_kernel) {
  const size_t rec = record_bytes(h->pitch);
  unsigned char* dst = const_cast<unsigned char*>(h->args.recv) + (t & 3) * (size_t)h->world * rec;
  *launched_kernel = false;
  if (!h->allreduce) return a->AllGather(h->args.send, dst, rec, kNcclUint8, h->comm, h->stream);
  ncclResult_t r = a->AllReduce(h->args.send, dst, 1, kNcclUint64, kNcclMin, h->comm, h->stream);
  if (r != 0) return r;
  if (launch_owner_row(h->args, h->stream) != cudaSuccess) return 1;  // reported as an NCCL failure
  *launched_kernel = true;
  return a->AllReduce(dst + 16, dst + 16, (size_t)h->pitch, kNcclUint32, kNcclSum, h->comm, h->stream);
}

// Exchange the records of iteration t (one per rank: its best candidate key
// and row) into recv slot t & 3 (NCCL: nccl_exchange; NVLink: already stored
// by the step kernels).  The next step kernel merges them in its
// prologue; `fold` additionally runs the select kernel so key_cur / G are
// final for the host (end of create, set_state and every pso_step call).
pso_status exchange(pso_swarm* h, uint64_t t, bool fold, bool into_local) {
  NvtxRange nvtx_range("gbest exchange");
  if (!h->xchg || h->colsplit) return PSO_OK;  // the column split exchanges inside its kernels
  if (h->args.p2p) {  // records travel by NVLink peer stores inside the kernels
    if (fold) {
      PSO_CUDA(h, launch_select(h->args, (unsigned)t, into_local, h->stream));
      ++h->launches;
    }
    return PSO_OK;
  }
  if (!h->comm) {
    h->poisoned = true;
    return fail(PSO_ERR_INVALID, "no communicator: enable the NVLink exchange before this call");
  }
  NcclApi* a = nccl();
  if (!a) {
    h->poisoned = true;
    return fail(PSO_ERR_NCCL, "NCCL unavailable");
  }
  bool kern = false;
  ncclResult_t r = nccl_exchange(h, a, t, &kern);
  if (kern) ++h->launches;
  if (r != 0) {
    h->poisoned = true;
    return fail(PSO_ERR_NCCL, "%s: %s", h->allreduce ? "ncclAllReduce exchange" : "ncclAllGather",
                nccl_str(r));
  }
  if (fold) {
    PSO_CUDA(h, launch_select(h->args, (unsigned)t, into_local, h->stream));
    ++h->launches;
  }
  return PSO_OK;
}

// Capture kGraphIters iterations of the NCCL exchange path starting at slot
// phase `phase` ([step kernel, nccl_exchange into recv slot (t & 3)] each) into
// an executable graph.  The step kernel reads its iteration from the control block,
// so the graph is valid for every start iteration with the same t & 3.  If the
// capture fails (e.g. NCCL without graph support) the handle stays eager.
pso_status capture_nccl_graph(pso_swarm* h, int phase) {
  NvtxRange nvtx_range("capture NCCL graph");
  NcclApi* a = nccl();
  if (!a || !h->comm) return PSO_OK;
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal);
  bool ok = e == cudaSuccess;
  for (int k = 0; ok && k < kGraphIters; ++k) {
    ok = launch_step(h->objective, h->args, h->cfg, h->stream) == cudaSuccess;
    bool kern = false;
    ok = ok && nccl_exchange(h, a, (uint64_t)((phase + k) & 3), &kern) == 0;
  }
  if (e == cudaSuccess) {
    cudaError_t e2 = cudaStreamEndCapture(h->stream, &g);
    ok = ok && e2 == cudaSuccess && g;
  }
  cudaGraphExec_t ex = nullptr;
  if (ok) ok = cudaGraphInstantiate(&ex, g, 0) == cudaSuccess;
  if (g) cudaGraphDestroy(g);
  cudaGetLastError();
  if (!ok) {
    if (ex) cudaGraphExecDestroy(ex);
    h->graph_off = true;
    return PSO_OK;
  }
  h->nccl_graph[phase] = ex;
  return PSO_OK;
}

pso_status sync_and_check(pso_swarm* h) {
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaStreamSynchronize");
  if (h->comm) {
    NcclApi* a = nccl();
    ncclResult_t ar = 0;
    if (a && a->CommGetAsyncError(h->comm, &ar) == 0 && ar != 0) {
      h->poisoned = true;
      return fail(PSO_ERR_NCCL, "NCCL async error: %s", nccl_str(ar));
    }
  }
  return PSO_OK;
}

// Reset the gbest control words before a full re-selection (create / set_state).
pso_status reset_ctl(pso_swarm* h, uint32_t t) {
  DevCtl c{};
  c.key_cur = ~0ull;
  c.key_acc = ~0ull;
  c.key_acc1 = ~0ull;
  c.improvements = 0;
  c.done = 0;
  c.t = t;
  c.bar_count = 0;
  h->args.t_base = t;  // async merges never reach back past the re-selection
  // improvements are preserved across set_state: read-modify-write
  DevCtl old{};
  PSO_CUDA(h, cudaMemcpyAsync(&old, h->args.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost, h->stream));
  PSO_CUDA(h, cudaStreamSynchronize(h->stream));
  c.improvements = old.improvements;
  PSO_CUDA(h, cudaMemcpyAsync(h->args.ctl, &c, sizeof(DevCtl), cudaMemcpyHostToDevice, h->stream));
  PSO_CUDA(h, cudaStreamSynchronize(h->stream));
  return PSO_OK;
}

// Sum the recorded step-kernel times into the totals (synchronises on them).
pso_status fold_events(pso_swarm* h) {
  for (size_t k = 0; k < h->events_used; ++k) {
    float ms = 0;
    PSO_CUDA(h, cudaEventSynchronize(h->events[k].stop));
    PSO_CUDA(h, cudaEventElapsedTime(&ms, h->events[k].start, h->events[k].stop));
    h->timed_ms += ms;
    h->timed_count += h->events[k].steps;
  }
  h->events_used = 0;
  return PSO_OK;
}

// Next event pair of the timing pool (bounded: folds into the totals when full).
pso_status next_event(pso_swarm* h, pso_swarm::Timed** out, uint64_t steps) {
  if (h->events_used == 4096) {
    pso_status st = fold_events(h);
    if (st != PSO_OK) return st;
  }
  if (h->events_used == h->events.size()) {
    pso_swarm::Timed e{};
    PSO_CUDA(h, cudaEventCreate(&e.start));
    PSO_CUDA(h, cudaEventCreate(&e.stop));
    h->events.push_back(e);
  }
  *out = &h->events[h->events_used++];
  (*out)->steps = steps;
  return PSO_OK;
}

// Per-dimension bounds [vlo | vhi | xlo | xhi] (4 x d host floats): finite,
// vlo_j <= vhi_j, xlo_j < xhi_j.
pso_status check_bounds(const float* b, int32_t d) {
  for (int32_t j = 0; j < d; ++j) {
    const float vlo = b[j], vhi = b[d + j], xlo = b[2 * d + j], xhi = b[3 * d + j];
    if (!std::isfinite(vlo) || !std::isfinite(vhi) || !std::isfinite(xlo) || !std::isfinite(xhi))
      return fail(PSO_ERR_INVALID, "bounds of dim %d are not finite", j);
    if (!(vlo <= vhi)) return fail(PSO_ERR_INVALID, "vlo > vhi at dim %d", j);
    if (!(xlo < xhi)) return fail(PSO_ERR_INVALID, "xlo >= xhi at dim %d", j);
  }
  return PSO_OK;
}

// Copy host bounds (dense d) into the pitched device table (padding 0).
pso_status upload_bounds(pso_swarm* h, const float* b) {
  std::vector<float> tab((size_t)4 * h->pitch, 0.f);
  for (int k = 0; k < 4; ++k)  // the column block [col_begin, col_begin + d_local)
    std::memcpy(&tab[(size_t)k * h->pitch], b + (size_t)k * h->d + h->col_begin,
                sizeof(float) * (size_t)h->d_local);
  PSO_CUDA(h, cudaMemcpyAsync(const_cast<float*>(h->args.bounds), tab.data(), tab.size() * 4,
                              cudaMemcpyHostToDevice, h->stream));
  PSO_CUDA(h, cudaStreamSynchronize(h->stream));
  return PSO_OK;
}

// Alg. 1 lines 1-3 + the first evaluation and best update (and, with an
// exchange, the first gbest exchange).
pso_status run_init(pso_swarm* h) {
  if (h->colsplit) {
    if (h->world > 1 && !h->args.p2p) {
      h->poisoned = true;
      return fail(PSO_ERR_INVALID, "column split with world > 1: enable the NVLink exchange first");
    }
    PSO_CUDA(h, launch_col_step(h->objective, h->args, h->cfg, 1, h->stream));
    PSO_CUDA(h, launch_col_decide(h->objective, h->args, h->cfg, 1, h->stream));
    h->launches += 2;
    pso_status st = sync_and_check(h);
    if (st != PSO_OK) return st;
    h->t = 0;
    h->inited = true;
    return PSO_OK;
  }
  if (h->n_local > 0) {
    PSO_CUDA(h, launch_init(h->objective, h->args, h->cfg, h->stream));
    ++h->launches;
  } else if (h->xchg) {  // no particles: publish a "no candidate" record of t = 0
    PSO_CUDA(h, launch_empty_step(h->args, 0, false, h->stream));
    ++h->launches;
  }
  pso_status st = exchange(h, 0, true, true);
  if (st != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  h->t = 0;
  h->inited = true;
  return PSO_OK;
}

float decode_fitness(unsigned long long key) {
  uint32_t o = (uint32_t)(key >> 32);
  uint32_t u = (o & 0x80000000u) ? (o & 0x7FFFFFFFu) : ~o;
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}

bool finite(float v) { return std::isfinite(v); }

}  // namespace

// ============================================================== C ABI
extern "C" {

const char* pso_status_string(pso_status s) {
  switch (s) {
    case PSO_OK: return "PSO_OK";
    case PSO_ERR_INVALID: return "PSO_ERR_INVALID";
    case PSO_ERR_NOMEM: return "PSO_ERR_NOMEM";
    case PSO_ERR_CUDA: return "PSO_ERR_CUDA";
    case PSO_ERR_NCCL: return "PSO_ERR_NCCL";
    case PSO_ERR_UNSUPPORTED: return "PSO_ERR_UNSUPPORTED";
    case PSO_ERR_POISONED: return "PSO_ERR_POISONED";
  }
  return "PSO_ERR_UNKNOWN";
}

const char* pso_last_error(void) { return g_last_error.c_str(); }

int pso_objective_registered(int32_t objective) { return objective_registered(objective) ? 1 : 0; }

pso_status pso_create(pso_handle* out, int64_t n, int32_t d, float w, float c1, float c2, float lo,
                      float hi, int32_t objective, uint64_t seed) {
  pso_opts o{};  // zero-initialised: defaults (current device, own stream, 1 GPU)
  return pso_create_ex(out, n, d, w, c1, c2, lo, hi, objective, seed, &o);
}

pso_status pso_create_ex(pso_handle* out, int64_t n, int32_t d, float w, float c1, float c2,
                         float lo, float hi, int32_t objective, uint64_t seed,
                         const pso_opts* opts) {
  NvtxRange nvtx_range("pso_create");
  if (!out) return fail(PSO_ERR_INVALID, "out is NULL");
  *out = nullptr;
  pso_opts o{};
  if (opts) o = *opts;
  // ---- validation (nothing touches the GPU before this passes)
  if (n < 1 || n >= (int64_t)1 << 32) return fail(PSO_ERR_INVALID, "n=%lld outside [1, 2^32)", (long long)n);
  if (d < 1) return fail(PSO_ERR_INVALID, "d=%d < 1", d);
  if (d > PSO_D_MAX) return fail(PSO_ERR_UNSUPPORTED, "d=%d > PSO_D_MAX=%d", d, PSO_D_MAX);
  bool colsplit = (o.flags & PSO_FLAG_COLUMN_SPLIT) != 0;
  if (d > PSO_D_MAX_ROW && !colsplit) {
    if (o.nccl_comm || o.world > 1)
      return fail(PSO_ERR_UNSUPPORTED, "d=%d > PSO_D_MAX_ROW=%d with a particle split: use "
                  "PSO_FLAG_COLUMN_SPLIT", d, PSO_D_MAX_ROW);
    colsplit = true;  // one GPU: rows longer than a cluster are tiled
  }
  // One GPU, rows that need a cluster of 4-16 CTAs: the column split (pbest
  // slots, G cache) is faster from d = 9728 up (Griewank 16384 x 16384: 806 ->
  // 708 us/iteration, 12288 x 10240: 482 -> 440; Rastrigin 12288 x 9728: 522
  // -> 484); at d <= 9216 the 4-CTA cluster stays (12288 x 9216: 473 vs 512).
  // PSO_CLUSTER (tuning) keeps the cluster.
  // PSO_COLSPLIT (tuning): 1 = the column split for any d, 0 = never automatically
  const char* cs = std::getenv("PSO_COLSPLIT");
  if (!colsplit && !o.nccl_comm && o.world <= 1 && d > PSO_D_AUTO_COLSPLIT && !std::getenv("PSO_CLUSTER") &&
      !(cs && *cs == '0'))
    colsplit = true;
  if (cs && *cs == '1' && !o.nccl_comm && o.world <= 1) colsplit = true;  // single GPU only
  if (colsplit && (o.flags & PSO_FLAG_ASYNC_GBEST))
    return fail(PSO_ERR_INVALID, "PSO_FLAG_COLUMN_SPLIT excludes PSO_FLAG_ASYNC_GBEST");
  if (!finite(w) || !finite(c1) || !finite(c2))
    return fail(PSO_ERR_INVALID, "w, c1, c2 must be finite");
  if ((c1 != 0.f && std::fabs(c1) < 0x1p-100f) || (c2 != 0.f && std::fabs(c2) < 0x1p-100f))
    return fail(PSO_ERR_UNSUPPORTED, "0 < |c1| or |c2| < 2^-100 is not supported");
  if (!finite(lo) || !finite(hi) || !(lo < hi))
    return fail(PSO_ERR_INVALID, "need finite lo < hi (got %g, %g)", lo, hi);
  if (!(o.vmax == o.vmax) || std::isinf(o.vmax)) return fail(PSO_ERR_INVALID, "vmax must be finite");
  if (!objective_registered(objective))
    return fail(PSO_ERR_INVALID, "objective %d is not registered", objective);
  if (o.flags & ~(uint32_t)(PSO_FLAG_TIMING | PSO_FLAG_DEFER_INIT | PSO_FLAG_ASYNC_GBEST |
                            PSO_FLAG_COLUMN_SPLIT | PSO_FLAG_DEVICE | PSO_FLAG_ALLREDUCE))
    return fail(PSO_ERR_INVALID, "unknown flags 0x%x", o.flags);
  if (o.bounds) {
    pso_status bs = check_bounds(o.bounds, d);
    if (bs != PSO_OK) return bs;
  }

  pso_swarm* h = new (std::nothrow) pso_swarm();
  if (!h) return fail(PSO_ERR_NOMEM, "host allocation failed");
  h->n = n;
  h->d = d;
  h->pitch = (d + 3) / 4 * 4;
  h->objective = objective;
  h->w = w;
  h->c1 = c1;
  h->c2 = c2;
  h->lo = lo;
  h->hi = hi;
  h->vmax = o.vmax > 0.f ? o.vmax : 1.0f;  // reading 3
  h->seed = seed;
  h->flags = o.flags;

  auto bail = [&](pso_status s) {
    pso_destroy(h);
    return s;
  };

  // ---- device and stream
  if ((o.flags & PSO_FLAG_DEVICE) && o.device < 0)
    return bail(fail(PSO_ERR_INVALID, "PSO_FLAG_DEVICE with device=%d < 0", o.device));
  if (o.flags & PSO_FLAG_DEVICE) {
    cudaError_t e = cudaSetDevice(o.device);
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaSetDevice"));
    h->device = o.device;
  } else {
    cudaError_t e = cudaGetDevice(&h->device);
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaGetDevice"));
    if ((e = cudaSetDevice(h->device)) != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaSetDevice"));
  }
  {
    cudaError_t e = cudaDeviceGetAttribute(&h->sm_count, cudaDevAttrMultiProcessorCount, h->device);
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaDeviceGetAttribute"));
    int major = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, h->device);
    if (major != 10)
      return bail(fail(PSO_ERR_UNSUPPORTED, "device %d has compute capability %d.x; this build is sm_100a only",
                       h->device, major));
  }
  if (o.stream) {
    h->stream = (cudaStream_t)o.stream;
  } else {
    cudaError_t e = cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaStreamCreate"));
    h->own_stream = true;
  }

  // ---- world (particle split)
  if (o.nccl_comm) {
    NcclApi* a = nccl();
    if (!a) return bail(fail(PSO_ERR_NCCL, "NCCL unavailable: %s", "dlopen failed"));
    h->comm = (ncclComm_t)o.nccl_comm;
    int cnt = 1, rk = 0;
    if (a->CommCount(h->comm, &cnt) != 0 || a->CommUserRank(h->comm, &rk) != 0)
      return bail(fail(PSO_ERR_NCCL, "ncclCommCount/UserRank failed"));
    h->world = cnt;
    h->rank = rk;
    const char* fx = std::getenv("PSO_FORCE_EXCHANGE");
    h->xchg = cnt > 1 || (fx && *fx && *fx != '0');
  } else if (o.world > 1) {  // ranks without a communicator: NVLink exchange only
    if (o.rank < 0 || o.rank >= o.world)
      return bail(fail(PSO_ERR_INVALID, "rank %d outside [0, %d)", o.rank, o.world));
    if (!(o.flags & PSO_FLAG_DEFER_INIT))
      return bail(fail(PSO_ERR_INVALID, "world > 1 without a communicator needs PSO_FLAG_DEFER_INIT "
                                        "(connect the NVLink exchange, then pso_init)"));
    h->world = o.world;
    h->rank = o.rank;
    h->xchg = true;
  }
  h->row_begin = (n * h->rank) / h->world;
  h->n_local = (n * (h->rank + 1)) / h->world - h->row_begin;
  h->d_local = d;
  int col_nvl = 0, col_q0 = 0, col_tile_f4 = 0, col_t0 = 0, col_nt = 0, col_nbt = 0;
  if (colsplit) {  // every rank: all rows, a block of whole column tiles (kernels.h col_tile)
    const int nvg = (d + 3) / 4;
    col_tile_f4 = col_tile(nvg);
    col_nbt = col_ntiles(nvg);
    if (col_nbt < h->world)
      return bail(fail(PSO_ERR_UNSUPPORTED, "column split: %d column tiles < world=%d (d too small)",
                       col_nbt, h->world));
    if (h->world > 1 && !(o.flags & PSO_FLAG_DEFER_INIT))
      return bail(fail(PSO_ERR_INVALID, "column split with world > 1 needs PSO_FLAG_DEFER_INIT "
                                        "(connect the NVLink exchange, then pso_init)"));
    h->colsplit = true;
    h->xchg = h->world > 1;
    h->row_begin = 0;
    h->n_local = n;
    col_rank_tiles(col_nbt, h->world, h->rank, &col_t0, &col_nt);
    col_q0 = col_t0 * col_tile_f4;
    col_nvl = std::min((col_t0 + col_nt) * col_tile_f4, nvg) - col_q0;
    h->col_begin = 4 * col_q0;
    h->d_local = std::min(4 * (col_q0 + col_nvl), d) - h->col_begin;
    h->pitch = 4 * col_nvl;
  }

  // ---- launch plan
  PlanHints hints;
  if (const char* v = std::getenv("PSO_VPT")) hints.vpt = std::atoi(v);
  if (const char* v = std::getenv("PSO_STAGES")) hints.stages = std::atoi(v);
  if (const char* v = std::getenv("PSO_CTAS")) hints.ctas = std::atoi(v);
  if (const char* v = std::getenv("PSO_CLUSTER")) hints.cluster = std::atoi(v);
  if (const char* v = std::getenv("PSO_GRAPH")) h->graph_off = *v == '0';
  if (const char* v = std::getenv("PSO_KERNEL")) {
    if (!std::strcmp(v, "reg")) hints.kernel = 0;
    if (!std::strcmp(v, "tma")) hints.kernel = 1;
  }
  if (colsplit) {
    cudaError_t e = plan_colsplit(objective, col_tile_f4, col_nt, n, h->sm_count,
                                  o.bounds != nullptr, &h->cfg);
    if (e == cudaErrorInvalidConfiguration) {
      cudaGetLastError();
      return bail(fail(PSO_ERR_UNSUPPORTED, "no column-split plan for d=%d", d));
    }
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "plan_colsplit"));
    const char* pdl = std::getenv("PSO_PDL");
    h->cfg.pdl = (pdl && *pdl == '0') ? 0 : 1;
  }
  if (!colsplit) {
    const char* v = std::getenv("PSO_RESIDENT");
    hints.allow_resident = !h->xchg && hints.kernel == -1 && !(v && !std::strcmp(v, "0"));
    if (const char* pv = std::getenv("PSO_PERSIST")) hints.persist = std::atoi(pv) ? 1 : 0;
    hints.bounds = o.bounds != nullptr;
  }
  if (!colsplit) {
    cudaError_t e = plan_launch(objective, d, h->n_local > 0 ? h->n_local : 1, h->sm_count,
                                hints, &h->cfg);
    if (e == cudaErrorInvalidConfiguration) {
      cudaGetLastError();
      return bail(fail(PSO_ERR_UNSUPPORTED, "no launch shape fits d=%d with the requested hints", d));
    }
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "plan_launch"));
    const char* pdl = std::getenv("PSO_PDL");
    h->cfg.pdl = (pdl && *pdl == '0') ? 0 : 1;
  }

  // ---- one arena: X, V, PB, pf, G, ctl, exchange records
  const size_t rows = (size_t)(h->n_local > 0 ? h->n_local : 1);
  const size_t mat = align_up(rows * (size_t)h->pitch * 4, 256);
  const size_t pfb = align_up(rows * 4, 256);
  const size_t gb = align_up((size_t)h->pitch * 4, 256);
  const size_t ctlb = align_up(sizeof(DevCtl), 256);
  const size_t boundb = o.bounds ? align_up(4 * (size_t)h->pitch * 4, 256) : 0;
  // lazy pbest rows on the TMA pipelines (step kernels that skip PB when PB == X)
  const char* lz = std::getenv("PSO_LAZY_PB");
  const bool lazy = colsplit ||  // the column split always defers pbest copies
                    (h->cfg.tma && !h->cfg.resident && !h->cfg.gridres && !(lz && *lz == '0'));
  const size_t pbxb = lazy ? align_up(rows, 256) : 0;
  const size_t rec = align_up(record_bytes(h->pitch), 256);
  // grid-resident kernel: [2 parities][grid] candidate rows, then their keys
  // grid-resident / persistent kernels: [2 parities][grid] candidate rows (+ keys for the former)
  const int cand_grid = h->cfg.gridres ? h->cfg.gridres_grid : h->cfg.persist ? h->cfg.persist_grid : 0;
  const size_t cand_rows = cand_grid ? align_up(2 * (size_t)cand_grid * h->pitch * 4, 256) : 0;
  const size_t candb = h->cfg.gridres ? cand_rows + align_up(2 * (size_t)h->cfg.gridres_grid * 8, 256) : cand_rows;
  const size_t sendb = (h->xchg && !colsplit) ? rec : 0;
  const size_t recvb = colsplit ? col_tag_bytes(h->world) + 2 * rows * (size_t)col_nbt * 16
                       : h->xchg ? 4 * (size_t)h->world * record_bytes(h->pitch) : 0;
  const bool async = (o.flags & PSO_FLAG_ASYNC_GBEST) != 0 && h->xchg;  // needs an exchange
  const size_t viewb = async ? gb : 0;  // the host's global gbest view
  // NVLink connect probe slots (pso_p2p_probe) after the receive area
  const size_t probeb = (recvb && h->xchg) ? align_up((size_t)h->world * 8, 256) : 0;
  h->arena_bytes = 3 * mat + pfb + gb + ctlb + boundb + pbxb + candb + viewb + sendb +
                   align_up(recvb, 256) + probeb;
  {
    cudaError_t e = cudaMalloc(&h->arena, h->arena_bytes);
    if (e == cudaErrorMemoryAllocation) {
      cudaGetLastError();
      return bail(fail(PSO_ERR_NOMEM, "cudaMalloc(%zu bytes) failed", h->arena_bytes));
    }
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaMalloc"));
  }
  unsigned char* p = (unsigned char*)h->arena;
  SwarmArgs& A = h->args;
  A.X = (float*)p; p += mat;
  A.V = (float*)p; p += mat;
  A.PB = (float*)p; p += mat;
  A.pf = (float*)p; p += pfb;
  A.G = (float*)p; p += gb;
  A.ctl = (DevCtl*)p; p += ctlb;
  A.bounds = o.bounds ? (const float*)p : nullptr; p += boundb;
  A.pbx = lazy ? p : nullptr; p += pbxb;
  A.lazy_pb = lazy ? 1 : 0;
  A.l2pf = 1;  // measured: C4 (all rows lazy) 547 -> 529 us; prefetching eager rows too slows NS
  if (const char* v = std::getenv("PSO_L2PF")) A.l2pf = std::atoi(v);
  if (A.l2pf < 0 || A.l2pf > 64) A.l2pf = 0;
  if (!lazy) A.l2pf = 0;
  if (colsplit) A.l2pf = 0;  // (an L2 prefetch of row tiles ahead measured slower: W16K 767 -> 847 us)
  if (const char* v = std::getenv("PSO_L2PF_ALL")) A.l2pf_all = std::atoi(v) != 0;
  // dynamic row claims (bit 0: streaming and column-split kernels; bit 1: the
  // cluster kernel, where they measured slower).  NS 628 -> 591 us, W64K 912 -> 878.
  A.dyn_rows = 1;
  if (const char* v = std::getenv("PSO_DYN_ROWS")) A.dyn_rows = std::atoi(v) & 3;
  A.serp = 1;  // measured: C3 36.9 -> 35.7 us (120 MB state, L2-borderline), NS / C4 within 1 %
  if (const char* v = std::getenv("PSO_SERP")) A.serp = std::atoi(v) != 0;
  A.cand = cand_grid ? (float*)p : nullptr;
  A.cand_key = h->cfg.gridres ? (unsigned long long*)(p + cand_rows) : nullptr;
  p += candb;
  A.G_view = async ? (float*)p : nullptr; p += viewb;
  A.async_gbest = async ? 1 : 0;
  A.send = sendb ? p : nullptr; p += sendb;
  A.recv = recvb ? p : nullptr;
  A.probe_off = align_up(recvb, 256);
  A.peer_timeout_ns = 60ull * 1000000000ull;  // PSO_PEER_TIMEOUT_S overrides (seconds)
  if (const char* v = std::getenv("PSO_PEER_TIMEOUT_S")) {
    const double sec = std::atof(v);
    if (sec > 0) A.peer_timeout_ns = (unsigned long long)(sec * 1e9);
  }
  A.n_local = h->n_local;
  A.row_begin = h->row_begin;
  A.d = d;
  A.nvec = h->pitch / 4;
  A.world = h->world;
  A.rank = h->rank;
  A.exchange = (h->xchg && !colsplit) ? 1 : 0;
  h->allreduce = (o.flags & PSO_FLAG_ALLREDUCE) != 0;
  A.xrecs = h->allreduce ? 1 : h->world;
  A.colsplit = colsplit ? 1 : 0;
  A.col_q0 = col_q0;
  A.nvec_glob = (d + 3) / 4;
  A.col_chunk = h->cfg.chunk;
  A.col_nb = col_nt;
  A.col_bbase = col_t0;
  A.col_nbt = col_nbt;
  A.w = w; A.c1 = c1; A.c2 = c2; A.lo = lo; A.hi = hi; A.vmax = h->vmax;
  A.seed_lo = (unsigned)seed;
  A.seed_hi = (unsigned)(seed >> 32);
  A.rk.set(seed);

  {
    cudaError_t e = cudaMemsetAsync(A.G, 0, gb + ctlb, h->stream);  // G and ctl
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaMemsetAsync"));
    if (sendb) e = cudaMemsetAsync(A.send, 0, sendb, h->stream);
    if (e == cudaSuccess && recvb)  // record tags that no iteration matches until written
      e = cudaMemsetAsync(const_cast<unsigned char*>(A.recv), 0xFF,
                          colsplit ? col_tag_bytes(h->world) : recvb, h->stream);
    if (e == cudaSuccess && probeb)
      e = cudaMemsetAsync(const_cast<unsigned char*>(A.recv) + A.probe_off, 0, probeb, h->stream);
    if (e != cudaSuccess) return bail(cuda_fail(nullptr, e, "cudaMemsetAsync"));
  }
  pso_status st = reset_ctl(h, 0);
  if (st != PSO_OK) return bail(st);
  if (o.bounds && (st = upload_bounds(h, o.bounds)) != PSO_OK) return bail(st);

  if (!(o.flags & PSO_FLAG_DEFER_INIT) && (st = run_init(h)) != PSO_OK) return bail(st);
  *out = h;
  return PSO_OK;
}

pso_status pso_init(pso_handle h) {
  NvtxRange nvtx_range("pso_init");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (h->inited) return fail(PSO_ERR_INVALID, "already initialised");
  if ((st = use_device(h)) != PSO_OK) return st;
  return run_init(h);
}

pso_status pso_step(pso_handle h, int64_t iters) {
  NvtxRange nvtx_range("pso_step");
  pso_status st = check_ready(h);
  if (st != PSO_OK) return st;
  if (iters < 0) return fail(PSO_ERR_INVALID, "iters=%lld < 0", (long long)iters);
  if (iters == 0) return PSO_OK;
  // the iteration counter is 32-bit on the device (Philox ctr[2], record tags)
  if (h->t + (uint64_t)iters >= ((uint64_t)1 << 32))
    return fail(PSO_ERR_UNSUPPORTED, "t=%llu + iters=%lld reaches 2^32 (32-bit iteration counter)",
                (unsigned long long)h->t, (long long)iters);
  if ((st = use_device(h)) != PSO_OK) return st;
  const bool timing = (h->flags & PSO_FLAG_TIMING) != 0;
  if (h->colsplit) {  // two kernels per iteration; the partials travel inside them
    // With PDL (default) the kernels overlap launch and drain, so one event pair
    // brackets the whole call: the timed "step kernel" is then k_col_step +
    // k_col_decide per iteration.  PSO_PDL=0: an event pair around each k_col_step.
    pso_swarm::Timed* call_ev = nullptr;
    if (timing && h->cfg.pdl) {
      if ((st = next_event(h, &call_ev, (uint64_t)iters)) != PSO_OK) return st;
      PSO_CUDA(h, cudaEventRecord(call_ev->start, h->stream));
    }
    for (int64_t it = 0; it < iters; ++it) {
      pso_swarm::Timed* ev = nullptr;
      if (timing && !call_ev && (st = next_event(h, &ev, 1)) != PSO_OK) return st;
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->start, h->stream));
      PSO_CUDA(h, launch_col_step(h->objective, h->args, h->cfg, 0, h->stream));
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->stop, h->stream));
      PSO_CUDA(h, launch_col_decide(h->objective, h->args, h->cfg, 0, h->stream));
      h->launches += 2;
    }
    if (call_ev) PSO_CUDA(h, cudaEventRecord(call_ev->stop, h->stream));
    h->t += (uint64_t)iters;
    return PSO_OK;
  }
  if (h->cfg.resident || h->cfg.gridres || h->cfg.persist) {  // the whole call is one launch
    for (int64_t done = 0; done < iters;) {
      const int chunk = (int)((iters - done) < (1 << 30) ? (iters - done) : (1 << 30));
      pso_swarm::Timed* ev = nullptr;
      if (timing && (st = next_event(h, &ev, (uint64_t)chunk)) != PSO_OK) return st;
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->start, h->stream));
      if (h->cfg.resident)
        PSO_CUDA(h, launch_resident(h->objective, h->args, h->cfg, chunk, h->stream));
      else if (h->cfg.persist)
        PSO_CUDA(h, launch_persist(h->objective, h->args, h->cfg, chunk, h->stream));
      else
        PSO_CUDA(h, launch_gridres(h->objective, h->args, h->cfg, chunk, h->stream));
      ++h->launches;
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->stop, h->stream));
      done += chunk;
    }
    h->t += (uint64_t)iters;
    return PSO_OK;
  }
  // With programmatic dependent launch the step kernels of consecutive
  // iterations overlap launch and drain, so an event between two of them would
  // serialise the pair: time the whole back-to-back run of the call instead
  // (per-launch average = its duration / iters).  A host-side exchange (NCCL)
  // sits between the launches anyway, so there every launch is timed alone.
  const bool per_call = timing && h->cfg.pdl && h->n_local > 0 && !(h->xchg && !h->args.p2p);
  pso_swarm::Timed* call_ev = nullptr;
  if (per_call) {
    if ((st = next_event(h, &call_ev, (uint64_t)iters)) != PSO_OK) return st;
    PSO_CUDA(h, cudaEventRecord(call_ev->start, h->stream));
  }
  const bool empty = h->n_local == 0;
  int64_t it = 0;
  // NCCL exchange: whole runs of kGraphIters iterations [step kernel, all-gather]
  // replay a captured CUDA graph (one per slot phase), so the host issues one
  // launch per kGraphIters iterations instead of 2 kGraphIters.
  if (!empty && !timing && h->xchg && !h->args.p2p && !h->graph_off) {
    while (iters - it > kGraphIters) {  // the last iteration stays eager (it folds)
      const int phase = (int)((h->t + (uint64_t)it + 1) & 3u);
      if (!h->nccl_graph[phase] && (st = capture_nccl_graph(h, phase)) != PSO_OK) return st;
      if (!h->nccl_graph[phase]) break;  // capture unavailable: eager from here on
      PSO_CUDA(h, cudaGraphLaunch(h->nccl_graph[phase], h->stream));
      h->launches += kGraphIters * (h->allreduce ? 2 : 1);  // step (+ owner-row) kernels
      it += kGraphIters;
    }
  }
  for (; it < iters; ++it) {
    const uint64_t ti = h->t + (uint64_t)it + 1;
    if (!empty) {
      pso_swarm::Timed* ev = nullptr;
      if (timing && !per_call && (st = next_event(h, &ev, 1)) != PSO_OK) return st;
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->start, h->stream));
      PSO_CUDA(h, launch_step(h->objective, h->args, h->cfg, h->stream));
      ++h->launches;
      if (ev) PSO_CUDA(h, cudaEventRecord(ev->stop, h->stream));
    } else if (h->xchg) {
      // A rank without particles runs no step kernel: k_empty_step publishes its
      // "no candidate" record (NVLink: after merging t - 1 as a prologue would).
      // Over NCCL nothing merges on this rank, so every iteration's records are
      // folded (a record only carries candidates strictly better than its
      // sender's incumbent: a gbest of an earlier iteration would otherwise
      // never reach this rank).
      PSO_CUDA(h, launch_empty_step(h->args, (unsigned)ti, true, h->stream));
      ++h->launches;
    }
    const bool fold = it + 1 == iters || (empty && !h->args.p2p);
    if ((st = exchange(h, ti, fold, empty)) != PSO_OK) return st;
  }
  if (call_ev) PSO_CUDA(h, cudaEventRecord(call_ev->stop, h->stream));
  h->t += (uint64_t)iters;
  return PSO_OK;
}

pso_status pso_synchronize(pso_handle h) {
  NvtxRange nvtx_range("pso_synchronize");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  return sync_and_check(h);
}

pso_status pso_get_gbest(pso_handle h, float* fitness, int64_t* index, float* pos) {
  NvtxRange nvtx_range("pso_get_gbest");
  pso_status st = check_ready(h);
  if (st != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  unsigned long long key = 0;
  // asynchronous gbest: the view folded at the end of the last call (every rank's records)
  const bool view = h->args.async_gbest != 0;
  const unsigned long long* ksrc = view ? &h->args.ctl->key_view : &h->args.ctl->key_cur;
  const float* gsrc = view ? h->args.G_view : h->args.G;
  PSO_CUDA(h, cudaMemcpyAsync(&key, ksrc, 8, cudaMemcpyDeviceToHost, h->stream));
  if (pos) PSO_CUDA(h, cudaMemcpyAsync(pos, gsrc, (size_t)h->d_local * 4, cudaMemcpyDeviceToHost, h->stream));
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  if (fitness) *fitness = decode_fitness(key);
  if (index) *index = (int64_t)(uint32_t)key;
  return PSO_OK;
}

pso_status pso_get_state(pso_handle h, float* x, float* v, float* pb, float* pf, uint64_t* t) {
  NvtxRange nvtx_range("pso_get_state");
  pso_status st = check_ready(h);
  if (st != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  const size_t w = (size_t)h->d_local * 4, sp = (size_t)h->pitch * 4, rows = (size_t)h->n_local;
  if (rows > 0) {
    // the plain layout first: deferred pbest rows (PB == X) written out; on the
    // column split also rows whose x lives in the PB array (swarm_colsplit.cuh)
    if (h->args.lazy_pb && (pb || (x && h->colsplit))) {
      PSO_CUDA(h, launch_materialize_pb(h->args, h->stream));
      ++h->launches;
    }
    if (x) PSO_CUDA(h, cudaMemcpy2DAsync(x, w, h->args.X, sp, w, rows, cudaMemcpyDeviceToHost, h->stream));
    if (v) PSO_CUDA(h, cudaMemcpy2DAsync(v, w, h->args.V, sp, w, rows, cudaMemcpyDeviceToHost, h->stream));
    if (pb) {
      PSO_CUDA(h, cudaMemcpy2DAsync(pb, w, h->args.PB, sp, w, rows, cudaMemcpyDeviceToHost, h->stream));
    }
    if (pf) PSO_CUDA(h, cudaMemcpyAsync(pf, h->args.pf, rows * 4, cudaMemcpyDeviceToHost, h->stream));
  }
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  if (t) *t = h->t;
  return PSO_OK;
}

pso_status pso_get_rows(pso_handle h, const int64_t* rows, int64_t m, float* x, float* v, float* pb,
                        float* pf) {
  NvtxRange nvtx_range("pso_get_rows");
  pso_status st = check_ready(h);
  if (st != PSO_OK) return st;
  if (m < 0 || (m > 0 && !rows)) return fail(PSO_ERR_INVALID, "bad rows / m");
  for (int64_t k = 0; k < m; ++k)
    if (rows[k] < 0 || rows[k] >= h->n_local)
      return fail(PSO_ERR_INVALID, "row %lld outside [0, %lld)", (long long)rows[k], (long long)h->n_local);
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  // lazy pbest rows (pbx bit 0: PB == x, not stored) read their pbest where x
  // is; column-split rows with pbx bit 1 hold x in PB and pb in X
  std::vector<unsigned char> lazy;
  if ((pb || x) && h->args.lazy_pb && m > 0) {
    lazy.resize((size_t)h->n_local);
    PSO_CUDA(h, cudaMemcpy(lazy.data(), h->args.pbx, lazy.size(), cudaMemcpyDeviceToHost));
  }
  const size_t w = (size_t)h->d_local * 4, sp = (size_t)h->pitch * 4;
  for (int64_t k = 0; k < m; ++k) {
    const size_t r = (size_t)rows[k], o = (size_t)k * h->d_local;
    const unsigned char fl = lazy.empty() ? 0 : lazy[r];
    const unsigned char* xr = reinterpret_cast<const unsigned char*>((fl & 2) ? h->args.PB : h->args.X) + r * sp;
    const unsigned char* pr = reinterpret_cast<const unsigned char*>((fl & 2) ? h->args.X : h->args.PB) + r * sp;
    if (x) PSO_CUDA(h, cudaMemcpyAsync(x + o, xr, w, cudaMemcpyDeviceToHost, h->stream));
    if (v)
      PSO_CUDA(h, cudaMemcpyAsync(v + o, reinterpret_cast<const unsigned char*>(h->args.V) + r * sp, w,
                                  cudaMemcpyDeviceToHost, h->stream));
    if (pb) PSO_CUDA(h, cudaMemcpyAsync(pb + o, (fl & 1) ? xr : pr, w, cudaMemcpyDeviceToHost, h->stream));
    if (pf) PSO_CUDA(h, cudaMemcpyAsync(pf + k, h->args.pf + r, 4, cudaMemcpyDeviceToHost, h->stream));
  }
  return sync_and_check(h);
}

pso_status pso_set_state(pso_handle h, const float* x, const float* v, const float* pb,
                         const float* pf, uint64_t t) {
  NvtxRange nvtx_range("pso_set_state");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (h->n_local > 0 && (!x || !v || !pb || !pf))
    return fail(PSO_ERR_INVALID, "set_state needs x, v, pb and pf");
  if (t >= ((uint64_t)1 << 32)) return fail(PSO_ERR_INVALID, "t=%llu >= 2^32", (unsigned long long)t);
  if ((st = use_device(h)) != PSO_OK) return st;
  const size_t w = (size_t)h->d_local * 4, sp = (size_t)h->pitch * 4, rows = (size_t)h->n_local;
  if (rows > 0) {
    const size_t mat = rows * sp;
    if (h->pitch != h->d_local) {  // zero the row padding
      PSO_CUDA(h, cudaMemsetAsync(h->args.X, 0, mat, h->stream));
      PSO_CUDA(h, cudaMemsetAsync(h->args.V, 0, mat, h->stream));
      PSO_CUDA(h, cudaMemsetAsync(h->args.PB, 0, mat, h->stream));
    }
    PSO_CUDA(h, cudaMemcpy2DAsync(h->args.X, sp, x, w, w, rows, cudaMemcpyHostToDevice, h->stream));
    PSO_CUDA(h, cudaMemcpy2DAsync(h->args.V, sp, v, w, w, rows, cudaMemcpyHostToDevice, h->stream));
    PSO_CUDA(h, cudaMemcpy2DAsync(h->args.PB, sp, pb, w, w, rows, cudaMemcpyHostToDevice, h->stream));
    PSO_CUDA(h, cudaMemcpyAsync(h->args.pf, pf, rows * 4, cudaMemcpyHostToDevice, h->stream));
    if (h->args.lazy_pb) PSO_CUDA(h, cudaMemsetAsync(h->args.pbx, 0, rows, h->stream));
  }
  if ((st = reset_ctl(h, (uint32_t)t)) != PSO_OK) return st;
  ++h->args.epoch;  // p2p: records written before this call can never match again
  // captured graphs hold the kernel parameters by value (epoch, t_base)
  for (cudaGraphExec_t& g : h->nccl_graph)
    if (g) cudaGraphExecDestroy(g), g = nullptr;
  if (rows > 0) {
    PSO_CUDA(h, launch_rebest(h->args, (unsigned)t, h->stream));
    ++h->launches;
  } else if (h->xchg) {  // no particles: a "no candidate" record of t (new epoch)
    PSO_CUDA(h, launch_empty_step(h->args, (unsigned)t, false, h->stream));
    ++h->launches;
  }
  if ((st = exchange(h, t, true, true)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  h->t = t;
  h->inited = true;
  return PSO_OK;
}

pso_status pso_set_bounds(pso_handle h, const float* bounds) {
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (!bounds) return fail(PSO_ERR_INVALID, "bounds is NULL");
  if (!h->args.bounds)
    return fail(PSO_ERR_UNSUPPORTED, "handle was created without per-dimension bounds");
  if ((st = check_bounds(bounds, h->d)) != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  return upload_bounds(h, bounds);
}

pso_status pso_p2p_handle(pso_handle h, void* ipc_handle, uint64_t* offset) {
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (!ipc_handle || !offset) return fail(PSO_ERR_INVALID, "ipc_handle/offset is NULL");
  if (!h->xchg) return fail(PSO_ERR_UNSUPPORTED, "handle has no exchange (no NCCL communicator)");
  if ((st = use_device(h)) != PSO_OK) return st;
  cudaIpcMemHandle_t mh;
  PSO_CUDA(h, cudaIpcGetMemHandle(&mh, h->arena));
  std::memcpy(ipc_handle, &mh, sizeof(mh));
  *offset = (uint64_t)((const unsigned char*)h->args.recv - (const unsigned char*)h->arena);
  return PSO_OK;
}

pso_status pso_p2p_connect(pso_handle h, const void* ipc_handles, const uint64_t* offsets) {
  NvtxRange nvtx_range("pso_p2p_connect");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (!ipc_handles || !offsets) return fail(PSO_ERR_INVALID, "ipc_handles/offsets is NULL");
  if (!h->xchg) return fail(PSO_ERR_UNSUPPORTED, "handle has no exchange (no NCCL communicator)");
  if (h->args.p2p) return fail(PSO_ERR_INVALID, "already connected");
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  if (h->peers_dev) return fail(PSO_ERR_INVALID, "already connected");
  // Failures here leave the handle usable (NCCL exchange): nothing is poisoned.
  auto undo = [&](cudaError_t e, const char* what) {
    for (void* p : h->ipc_opened) cudaIpcCloseMemHandle(p);
    h->ipc_opened.clear();
    if (h->peers_dev) cudaFree(h->peers_dev);
    h->peers_dev = nullptr;
    return cuda_fail(nullptr, e, what);
  };
  std::vector<unsigned char*> peers((size_t)h->world);
  for (int r = 0; r < h->world; ++r) {
    if (r == h->rank) {  // our own receive buffer
      peers[r] = const_cast<unsigned char*>(h->args.recv);
      continue;
    }
    cudaIpcMemHandle_t mh;
    std::memcpy(&mh, (const unsigned char*)ipc_handles + (size_t)r * sizeof(mh), sizeof(mh));
    void* base = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&base, mh, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return undo(e, "cudaIpcOpenMemHandle");
    h->ipc_opened.push_back(base);
    peers[r] = (unsigned char*)base + offsets[r];
  }
  cudaError_t e = cudaMalloc(&h->peers_dev, sizeof(unsigned char*) * peers.size());
  if (e != cudaSuccess) return undo(e, "cudaMalloc");
  e = cudaMemcpy(h->peers_dev, peers.data(), sizeof(unsigned char*) * peers.size(),
                 cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return undo(e, "cudaMemcpy");
  h->args.peers = (unsigned char* const*)h->peers_dev;
  return PSO_OK;
}

pso_status pso_p2p_probe(pso_handle h, int32_t phase, int32_t* ok) {
  NvtxRange nvtx_range("pso_p2p_probe");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (phase != 0 && phase != 1) return fail(PSO_ERR_INVALID, "phase must be 0 or 1");
  if (phase == 1 && !ok) return fail(PSO_ERR_INVALID, "ok is NULL");
  if (!h->peers_dev) return fail(PSO_ERR_INVALID, "pso_p2p_connect first");
  if ((st = use_device(h)) != PSO_OK) return st;
  int* dev_ok = nullptr;
  if (phase == 1) PSO_CUDA(h, cudaMalloc(&dev_ok, sizeof(int)));
  cudaError_t e = launch_p2p_probe(h->args, phase, dev_ok, h->stream);
  int host_ok = 0;
  if (e == cudaSuccess && phase == 1)
    e = cudaMemcpyAsync(&host_ok, dev_ok, sizeof(int), cudaMemcpyDeviceToHost, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (dev_ok) cudaFree(dev_ok);
  if (e != cudaSuccess) return cuda_fail(h, e, "p2p probe");
  if (phase == 1) *ok = host_ok;
  return PSO_OK;
}

pso_status pso_p2p_enable(pso_handle h, int32_t on) {
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if (on && !h->peers_dev) return fail(PSO_ERR_INVALID, "pso_p2p_connect first");
  if (!on && h->colsplit)
    return fail(PSO_ERR_UNSUPPORTED, "the column split exchanges only over NVLink");
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  h->args.p2p = on ? 1 : 0;
  h->args.xrecs = (on || !h->allreduce) ? h->world : 1;
  for (cudaGraphExec_t& g : h->nccl_graph)  // captured with the previous exchange's arguments
    if (g) cudaGraphExecDestroy(g), g = nullptr;
  return PSO_OK;
}

pso_status pso_get_info(pso_handle h, pso_info* info) {
  if (!h) return fail(PSO_ERR_INVALID, "NULL handle");
  if (!info) return fail(PSO_ERR_INVALID, "info is NULL");
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  if ((st = fold_events(h)) != PSO_OK) return st;
  DevCtl c{};
  PSO_CUDA(h, cudaMemcpy(&c, h->args.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost));
  std::memset(info, 0, sizeof(*info));
  info->n = h->n;
  info->n_local = h->n_local;
  info->row_begin = h->row_begin;
  info->d = h->d;
  info->pitch = h->pitch;
  info->rank = h->rank;
  info->world = h->world;
  info->threads_per_cta = h->cfg.threads;
  info->vec_per_thread = h->cfg.vpt;
  info->grid = h->cfg.grid;
  info->ctas_per_sm = h->cfg.ctas_per_sm;
  info->tma_pipeline = h->cfg.tma;
  info->pipeline_stages = h->cfg.stages;
  info->smem_bytes = (int32_t)(h->cfg.resident ? h->cfg.resident_smem : h->cfg.smem);
  info->resident = h->cfg.resident ? 1 : h->cfg.gridres ? 2 : h->cfg.persist ? 3 : 0;
  info->bounds = h->args.bounds ? 1 : 0;
  info->cluster = h->cfg.cluster;
  if (h->cfg.resident) {
    info->threads_per_cta = h->cfg.resident_threads;
    info->grid = 1;
  }
  if (h->cfg.gridres) {
    info->threads_per_cta = h->cfg.compute;
    info->grid = h->cfg.gridres_grid;
    info->smem_bytes = (int32_t)h->cfg.gridres_smem;
  }
  if (h->cfg.persist) info->grid = h->cfg.persist_grid;
  info->vmax = h->vmax;
  info->t = h->t;
  info->launches = h->launches;
  info->improvements = c.improvements;
  info->pb_loads = c.pb_loads;
  info->pb_stores = c.pb_stores;
  info->lazy_pb = h->args.lazy_pb;
  info->step_kernel_ms = h->timed_ms;
  info->step_kernel_count = h->timed_count;
  info->column_split = h->colsplit ? 1 : 0;
  info->col_begin = h->col_begin;
  info->d_local = h->d_local;
  info->col_tiles = h->args.col_nbt;
  info->arena_bytes = h->arena_bytes;
  return PSO_OK;
}

pso_status pso_reset_counters(pso_handle h) {
  pso_status st = check_handle(h);
  if (st != PSO_OK) return st;
  if ((st = use_device(h)) != PSO_OK) return st;
  if ((st = sync_and_check(h)) != PSO_OK) return st;
  h->launches = 0;
  h->timed_ms = 0;
  h->timed_count = 0;
  h->events_used = 0;
  unsigned long long zero[2] = {0, 0};
  PSO_CUDA(h, cudaMemcpy(&h->args.ctl->improvements, zero, 8, cudaMemcpyHostToDevice));
  PSO_CUDA(h, cudaMemcpy(&h->args.ctl->pb_loads, zero, 16, cudaMemcpyHostToDevice));
  return PSO_OK;
}

void pso_destroy(pso_handle h) {
  if (!h) return;
  cudaSetDevice(h->device);
  if (h->stream) cudaStreamSynchronize(h->stream);
  for (auto& e : h->events) {
    cudaEventDestroy(e.start);
    cudaEventDestroy(e.stop);
  }
  for (cudaGraphExec_t g : h->nccl_graph)
    if (g) cudaGraphExecDestroy(g);
  for (void* p : h->ipc_opened) cudaIpcCloseMemHandle(p);
  if (h->peers_dev) cudaFree(h->peers_dev);
  if (h->arena) cudaFree(h->arena);
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  cudaGetLastError();
  delete h;
}

// ------------------------------------------------------------ NCCL helpers
pso_status pso_nccl_get_unique_id(void* id128) {
  if (!id128) return fail(PSO_ERR_INVALID, "id is NULL");
  NcclApi* a = nccl();
  if (!a) return fail(PSO_ERR_NCCL, "NCCL unavailable");
  ncclUniqueId id;
  ncclResult_t r = a->GetUniqueId(&id);
  if (r != 0) return fail(PSO_ERR_NCCL, "ncclGetUniqueId: %s", nccl_str(r));
  std::memcpy(id128, &id, sizeof(id));
  return PSO_OK;
}

pso_status pso_nccl_comm_init(void** comm, int32_t nranks, const void* id128, int32_t rank,
                              int32_t device) {
  if (!comm || !id128) return fail(PSO_ERR_INVALID, "comm/id is NULL");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail(PSO_ERR_INVALID, "bad rank/nranks");
  NcclApi* a = nccl();
  if (!a) return fail(PSO_ERR_NCCL, "NCCL unavailable");
  if (device >= 0) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaSetDevice");
  }
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof(id));
  ncclComm_t c = nullptr;
  ncclResult_t r = a->CommInitRank(&c, nranks, id, rank);
  if (r != 0) return fail(PSO_ERR_NCCL, "ncclCommInitRank: %s", nccl_str(r));
  *comm = c;
  return PSO_OK;
}

pso_status pso_nccl_comm_destroy(void* comm) {
  if (!comm) return PSO_OK;
  NcclApi* a = nccl();
  if (!a) return fail(PSO_ERR_NCCL, "NCCL unavailable");
  ncclResult_t r = a->CommDestroy((ncclComm_t)comm);
  if (r != 0) return fail(PSO_ERR_NCCL, "ncclCommDestroy: %s", nccl_str(r));
  return PSO_OK;
}

// ------------------------------------------------------------ debug entry points
pso_status pso_debug_philox(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j0,
                            int64_t m, uint32_t* out, int32_t use_curand, int32_t device) {
  if (m < 0 || (m > 0 && !out)) return fail(PSO_ERR_INVALID, "bad m/out");
  if (m == 0) return PSO_OK;
  if (device >= 0) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaSetDevice");
  }
  unsigned* dev = nullptr;
  cudaError_t e = cudaMalloc(&dev, (size_t)m * 4);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaMalloc");
  e = debug_philox(seed, tag, t, i, j0, m, dev, use_curand, 0);
  if (e == cudaSuccess) e = cudaMemcpy(out, dev, (size_t)m * 4, cudaMemcpyDeviceToHost);
  cudaFree(dev);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "debug_philox");
  return PSO_OK;
}

pso_status pso_debug_objective(int32_t objective, const float* X, int64_t m, int32_t d, float* out,
                               int32_t device) {
  if (m < 0 || d < 1 || d > PSO_D_MAX || (m > 0 && (!X || !out)))
    return fail(PSO_ERR_INVALID, "bad arguments");
  if (!objective_registered(objective)) return fail(PSO_ERR_INVALID, "objective %d not registered", objective);
  if (m == 0) return PSO_OK;
  if (device >= 0) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaSetDevice");
  }
  int dev_id = 0, sms = 148;
  cudaGetDevice(&dev_id);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev_id);
  const int pitch = (d + 3) / 4 * 4;
  float* dX = nullptr;
  float* dO = nullptr;
  cudaError_t e = cudaMalloc(&dX, (size_t)m * pitch * 4);
  if (e == cudaSuccess) e = cudaMalloc(&dO, (size_t)m * 4);
  if (e == cudaSuccess) e = cudaMemset(dX, 0, (size_t)m * pitch * 4);
  if (e == cudaSuccess)
    e = cudaMemcpy2D(dX, (size_t)pitch * 4, X, (size_t)d * 4, (size_t)d * 4, (size_t)m,
                     cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = debug_objective(objective, dX, m, d, pitch, dO, sms, 0);
  if (e == cudaSuccess) e = cudaMemcpy(out, dO, (size_t)m * 4, cudaMemcpyDeviceToHost);
  cudaFree(dX);
  cudaFree(dO);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "debug_objective");
  return PSO_OK;
}

}  // extern "C"
