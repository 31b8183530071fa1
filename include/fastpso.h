/*
 * fastpso.h — C ABI of the B200-native FastPSO hot path.
 *
 * The library runs the per-iteration swarm update of FastPSO (Liu, Wen, Cai,
 * ICPP'21) as ONE fused sm_100a kernel per iteration: counter-based random
 * weights, the velocity/position update, the objective evaluation, the pbest
 * compare-and-copy and the gbest argmin.  Citations are PAPER.md lines (P:Lnnn):
 *
 *   Alg. 1, P:L81-103   inputs n, omega, c1, c2, max_iter; output "the optimal
 *                       positions of the particles"
 *   Eq. 1,  P:L105-109  v' = omega v + c1 l (.) (pbest - p) + c2 g (.) (gbest - p)
 *   Eq. 2,  P:L111-115  p' = p + v'
 *   Eq. 4,  P:L171-253  the same on the n x d matrices V, P, L, G, E_l, E_g
 *   Eq. 5,  P:L255-265  user-defined velocity bounds (here: |v| <= vmax)
 *   Sec 3.1 P:L135      random swarm initialisation and per-iteration L, G
 *   Sec 3.2 P:L137-147  swarm evaluation; user-defined evaluation schema
 *   Sec 3.3 P:L149-153  pbest update; gbest = min and its index by reduction
 *   P:L281              multi-GPU by particle splitting (made synchronous here)
 *   P:L667              one cached device allocation (one arena per handle)
 *
 * Conventions (all entry points):
 *   - Every call returns a pso_status; nothing aborts or throws across the ABI.
 *     pso_last_error() gives a thread-local detail string for the last failure.
 *   - Host buffers are owned by the caller, dense row-major (rows of d floats,
 *     no padding).  Device memory is owned by the handle (one arena).
 *   - pso_step only enqueues work on the handle's stream.  Launch errors are
 *     returned at once; asynchronous faults surface at the next synchronising
 *     call (pso_get_gbest / pso_get_state / pso_get_info / pso_synchronize).
 *   - After any CUDA or NCCL error the handle is POISONED: every later call
 *     except pso_destroy returns PSO_ERR_POISONED.
 *   - A handle is not thread-safe; different handles are independent.
 *   - Multi-GPU (opts.nccl_comm != NULL, world k > 1): n is the GLOBAL swarm
 *     size, rank r owns global rows [floor(n r / k), floor(n (r+1) / k)).  All
 *     calls except get_* / destroy are collective: every rank must make the
 *     same sequence.  The gbest is bitwise identical on every rank, and every
 *     result is bitwise independent of k.
 *   - Determinism: the same arguments and seed give bitwise identical results;
 *     pso_step(h, a); pso_step(h, b) is bitwise pso_step(h, a + b).
 *   - Numerics: fp32 state; the update (Eq. 1, 5, 2) is evaluated in the fixed
 *     order a = w*v; b = (c1*r1)*(pb-x); c = (c2*r2)*(g-x); v' = (a+b)+c,
 *     v' = clamp(v', -vmax, vmax), x' = clamp(x + v', lo, hi), each op rounded
 *     once (no FMA contraction).  Fitness is fp32 (tree-reduced per particle).
 */
#ifndef FASTPSO_H
#define FASTPSO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FASTPSO_VERSION_MAJOR 0
#define FASTPSO_VERSION_MINOR 1
#define PSO_D_MAX_ROW 65536 /* max dimension of the row kernels: <= 8192 one CTA per row;
                              above, a thread-block cluster of up to 16 CTAs per row (a
                              single GPU switches to the column split above
                              PSO_D_AUTO_COLSPLIT) */
#define PSO_D_MAX (1 << 24) /* max dimension: above PSO_D_MAX_ROW the column split
                              (PSO_FLAG_COLUMN_SPLIT) is used on a single GPU */
#define PSO_D_AUTO_COLSPLIT 9216 /* a single-GPU handle (no communicator, world <= 1)
                              with d above this uses the column split: faster than
                              the 4-16-CTA clusters per row from d = 9728 up (W16K
                              16384^2: 708 vs 806 us) */

typedef struct pso_swarm* pso_handle; /* opaque; owns all device memory */

typedef enum {
  PSO_OK = 0,
  PSO_ERR_INVALID = 1,     /* bad argument (nothing was changed) */
  PSO_ERR_NOMEM = 2,       /* device (or host) allocation failed */
  PSO_ERR_CUDA = 3,        /* CUDA runtime error (handle is poisoned) */
  PSO_ERR_NCCL = 4,        /* NCCL error or NCCL unavailable (poisoned) */
  PSO_ERR_UNSUPPORTED = 5, /* valid but not supported (e.g. d > PSO_D_MAX) */
  PSO_ERR_POISONED = 6     /* an earlier CUDA/NCCL error poisoned the handle */
} pso_status;

/* Objectives (Sec 3.2).  Definitions (k = 1..d):
 *   SPHERE      sum x_k^2
 *   RASTRIGIN   sum (x_k^2 + 10 - 10 cos(2 pi x_k))               ([20])
 *   ROSENBROCK  sum_{k<d} 100 (x_{k+1} - x_k^2)^2 + (x_k - 1)^2   ([20])
 *   GRIEWANK    1 + sum x_k^2 / 4000 - prod cos(x_k / sqrt(k))
 *   ACKLEY      -20 exp(-0.2 sqrt(sum x^2/d)) - exp(sum cos(2 pi x)/d) + 20 + e
 *               ([20]); compiled through the user-functor schema
 *               (csrc/user_objectives.cuh), as a user objective would be
 *   EASOM       -(-1)^d prod cos^2(x_k) exp(-sum (x_k - pi)^2)
 * Ids >= PSO_OBJ_CUSTOM_BASE are user functors registered at compile time in
 * csrc/user_objectives.cuh (the paper's evaluation_kernel<L> schema,
 * P:L139-145, realised as compile-time device functors). */
enum {
  PSO_OBJ_SPHERE = 1,
  PSO_OBJ_RASTRIGIN = 2,
  PSO_OBJ_ROSENBROCK = 3,
  PSO_OBJ_GRIEWANK = 4,
  PSO_OBJ_ACKLEY = 5,
  PSO_OBJ_EASOM = 6,
  PSO_OBJ_CUSTOM_BASE = 64
};

/* Option flags. */
enum {
  PSO_FLAG_TIMING = 1,     /* record CUDA events around every step kernel launch;
                              totals are reported by pso_get_info */
  PSO_FLAG_DEFER_INIT = 2,  /* allocate and plan only; pso_init runs Alg. 1 lines 1-3
                              (lets ranks connect the NVLink exchange first) */
  PSO_FLAG_ASYNC_GBEST = 4, /* NEXT-4, "updated in an asynchronous manner": each
                              rank's step kernel adopts its own candidates at once and
                              merges its peers' records one iteration late, so no rank
                              waits for the iteration its peers are in.  Deterministic
                              for a given world size, but results depend on it; with
                              world = 1 identical to the synchronous mode.
                              pso_get_gbest returns the global view folded from every
                              rank's records at the end of the last pso_step call. */
  PSO_FLAG_ALLREDUCE = 32,  /* NCCL exchange as north_star states it:
                              per iteration an ncclAllReduce(min) of the u64 packed
                              (fitness, index) keys, then the owning rank's candidate
                              row is broadcast bit-exactly by an ncclAllReduce(sum) of
                              the row as u32 words to which every other rank adds
                              zeros (root decided on the device, no host sync).
                              Default: one ncclAllGather of the (key, row) records.
                              Either is replaced by the NVLink peer exchange once
                              pso_p2p_enable(h, 1) succeeds. */
  PSO_FLAG_DEVICE = 16,     /* use pso_opts.device as the CUDA ordinal; without it the
                              handle runs on the caller's current device (so a
                              zero-initialised pso_opts means "defaults") */
  PSO_FLAG_COLUMN_SPLIT = 8 /* NEXT-3, "tile matrix": every rank holds ALL n
                              particles but only a block of the columns.  Rows are cut
                              into column tiles of T = clamp(ceil(nv / 8), 32, 512)
                              float4 (nv = ceil(d / 4)); rank r owns tiles
                              [floor(nt r / world), floor(nt (r+1) / world)) of the nt
                              (dims [col_begin, col_begin + d_local), pso_get_info).
                              Each iteration: the move of the block + per-tile fitness
                              partials stored into every rank's partial table over
                              NVLink; then every rank combines the partials of each row
                              in tile order, decides pbest / gbest identically, and
                              keeps its block of G.  The tiling depends on d only, so
                              results are bitwise the same for every world size.  State calls (get/set_state,
                              get_gbest) read and write the rank's column block (n x
                              d_local; pf has all n rows and must be the same on every
                              rank).  world > 1 needs the NVLink exchange (p2p connect +
                              enable before pso_init, so PSO_FLAG_DEFER_INIT) and
                              nt >= world.  Chosen automatically for a single
                              GPU when d > PSO_D_AUTO_COLSPLIT (unless the PSO_CLUSTER
                              tuning variable asks for a cluster).  Not with ASYNC_GBEST. */
};

/* Options; a zero-initialised struct means "defaults". */
typedef struct {
  float vmax;      /* Eq. 5 bound |v| <= vmax; <= 0 -> 1.0 (reading 3) */
  int32_t device;  /* CUDA ordinal, read only with PSO_FLAG_DEVICE (else the
                      caller's current device is used) */
  void* stream;    /* cudaStream_t to enqueue on; NULL -> a library-owned stream */
  void* nccl_comm; /* ncclComm_t (see pso_nccl_comm_init); NULL -> single GPU */
  uint32_t flags;  /* PSO_FLAG_* */
  int32_t world, rank; /* without nccl_comm: world > 1 ranks that exchange only over
                          NVLink (needs PSO_FLAG_DEFER_INIT: create, p2p connect +
                          enable, then pso_init); ignored with a communicator */
  const float* bounds; /* NULL, or 4*d host floats [vlo | vhi | xlo | xhi]: per-dimension
                          velocity bounds (Eq. 5: lower/upper_bound_j) and
                          domain (x clamp); replaces vmax / lo / hi (which must still be
                          valid).  Init draws x0 ~ U[xlo_j, xhi_j], v0 ~ U[vlo_j, vhi_j].
                          Needs finite values, vlo_j <= vhi_j, xlo_j < xhi_j. */
} pso_opts;

/* Create a swarm of n particles in d dimensions and initialise it (Alg. 1
 * lines 1-3, Sec 3.1): x0 ~ U[lo, hi], v0 ~ U[-vmax, vmax] from the Philox
 * streams keyed on (seed, particle, dim); the first evaluation; pbest = x0;
 * gbest = the lowest index attaining min f(x0).
 *   out        receives the handle (set to NULL on failure)
 *   n          global swarm size, 1 <= n < 2^32
 *   d          dimension, 1 <= d <= PSO_D_MAX (else PSO_ERR_UNSUPPORTED); a
 *              particle-split handle (world > 1 without PSO_FLAG_COLUMN_SPLIT)
 *              needs d <= PSO_D_MAX_ROW
 *   w, c1, c2  Eq. 1 parameters, finite; c1, c2 = 0 or |c| >= 2^-100 (else
 *              PSO_ERR_UNSUPPORTED: the kernel folds the 2^-24 of the uniform
 *              into c, exact only away from the subnormal range)
 *   lo < hi    finite domain bounds; positions are clamped to [lo, hi]
 *   objective  PSO_OBJ_* or a registered custom id (else PSO_ERR_INVALID)
 *   seed       64-bit Philox key
 * Blocks until initialisation has completed (errors are reported here). */
pso_status pso_create(pso_handle* out, int64_t n, int32_t d, float w, float c1, float c2,
                      float lo, float hi, int32_t objective, uint64_t seed);
pso_status pso_create_ex(pso_handle* out, int64_t n, int32_t d, float w, float c1, float c2,
                         float lo, float hi, int32_t objective, uint64_t seed,
                         const pso_opts* opts);

/* Run the deferred initialisation of a handle created with PSO_FLAG_DEFER_INIT
 * (Alg. 1 lines 1-3 + the first evaluation and gbest).  Collective.  Every
 * other call except pso_set_state, pso_get_info, the p2p calls and destroy
 * needs an initialised swarm (else PSO_ERR_INVALID). */
pso_status pso_init(pso_handle h);

/* Enqueue iters >= 0 iterations; each is one fused kernel: move (Eq. 1, 5,
 * 2), evaluate (Sec 3.2), pbest (Sec 3.3, strict <) and gbest (strict <,
 * lowest index among equal new minima).  Tiny and shared-memory-sized swarms
 * on one GPU run the whole call as one launch (pso_info.resident).
 * world > 1 (particle split): with the NVLink exchange (pso_p2p_*)
 * the same kernel stores the rank's (key, candidate row) record into every
 * rank over NVLink and the next iteration's kernel merges them, so an
 * iteration is still one kernel; one select kernel per call folds the last
 * records for the host.  With the NCCL fallback each iteration adds an
 * ncclAllGather of the records (runs of 4 iterations are replayed as a
 * captured CUDA graph).  A rank without particles runs a one-warp record
 * kernel per iteration instead of the step kernel.  The column split
 * (PSO_FLAG_COLUMN_SPLIT) runs two kernels per iteration.
 * PSO_ERR_UNSUPPORTED if the iteration counter would reach 2^32 (it is the
 * 32-bit Philox counter word t). */
pso_status pso_step(pso_handle h, int64_t iters);

/* Wait for all enqueued work and report asynchronous errors. */
pso_status pso_synchronize(pso_handle h);

/* Synchronise and read the global best: fitness, global particle index, and
 * (if pos != NULL) its d-float position.  Any output pointer may be NULL.
 * Host pointers.  Identical bits on every rank. */
pso_status pso_get_gbest(pso_handle h, float* fitness, int64_t* index, float* pos);

/* Synchronise and copy the rank-local state to host buffers (any may be NULL):
 * x, v, pb: n_local x d floats; pf: n_local floats; t: iterations done. */
pso_status pso_get_state(pso_handle h, float* x, float* v, float* pb, float* pf, uint64_t* t);

/* Synchronise and copy m rank-local rows (local indices rows[k] in [0, n_local);
 * row k is particle row_begin + rows[k]) to host buffers (any may be NULL):
 * x, v, pb: m x d floats; pf: m floats.  The state is not changed (a pbest
 * deferred by the lazy rows is read from x; on the column split each row is
 * read from the slot that holds it).  For sampling swarms too large
 * to copy whole (e.g. 2.9M x 4096: 142 GB).  PSO_ERR_INVALID for an index
 * outside [0, n_local) or m < 0. */
pso_status pso_get_rows(pso_handle h, const int64_t* rows, int64_t m, float* x, float* v, float* pb,
                        float* pf);

/* Replace the rank-local state from host buffers (all required: x, v, pb are
 * n_local x d, pf is n_local; NaN pf is read as +inf) and set the iteration
 * counter to t.  The gbest is recomputed from pf/pb exactly as after create.
 * Collective when world > 1.  Synchronous. */
pso_status pso_set_state(pso_handle h, const float* x, const float* v, const float* pb,
                         const float* pf, uint64_t t);

/* Replace the per-dimension bounds (same layout as pso_opts.bounds) of a
 * handle created with bounds; applies to the following iterations.
 * PSO_ERR_UNSUPPORTED for a handle created with scalar bounds.  Synchronous. */
pso_status pso_set_bounds(pso_handle h, const float* bounds);

/* Information and counters. */
typedef struct {
  int64_t n, n_local, row_begin; /* global size, local rows, first global row */
  int32_t d, pitch;              /* dimension, row pitch in floats (16-B rows) */
  int32_t rank, world;
  int32_t threads_per_cta, vec_per_thread, grid, ctas_per_sm;
  int32_t tma_pipeline;          /* 1: bulk-copy (TMA) pipelined step kernel */
  int32_t pipeline_stages;       /* rows in flight per CTA in that pipeline */
  int32_t smem_bytes;            /* dynamic shared memory of the step kernel */
  int32_t resident;              /* 0: streaming kernel, one launch per iteration;
                                    1: tiny swarm held in one CTA's shared memory,
                                    2: swarm held in the whole grid's shared memory
                                    (cooperative launch), 3: persistent streaming
                                    kernel (rows streamed from HBM every iteration,
                                    a grid barrier per iteration; opt-in with the
                                    PSO_PERSIST=1 tuning variable); 1-3 run a whole
                                    pso_step call in one launch (single GPU only) */
  int32_t bounds;                /* 1: per-dimension bounds in use */
  int32_t cluster;               /* > 0: each row is split in column blocks over a
                                    thread-block cluster of this many CTAs (d > 8192) */
  float vmax;
  uint64_t t;                    /* iterations done */
  uint64_t launches;             /* kernels launched by this handle so far */
  uint64_t improvements;         /* pbest improvements (rows) so far, all steps */
  uint64_t pb_loads;             /* streaming kernels: pbest rows read from memory */
  uint64_t pb_stores;            /* streaming kernels: pbest rows written to memory */
  int32_t lazy_pb;               /* 1: rows whose pbest equals x skip the pb load/store */
  double step_kernel_ms;         /* PSO_FLAG_TIMING: summed step-kernel time */
  uint64_t step_kernel_count;    /* PSO_FLAG_TIMING: step kernels timed */
  size_t arena_bytes;            /* device bytes owned by the handle */
  int32_t column_split;          /* 1: PSO_FLAG_COLUMN_SPLIT layout (NEXT-3) */
  int32_t col_begin, d_local;    /* the rank's column block: dims [col_begin,
                                    col_begin + d_local) (0, d without the split) */
  int32_t col_tiles;             /* column split: tiles per row over all ranks */
} pso_info;
pso_status pso_get_info(pso_handle h, pso_info* info);
/* Reset launches / improvements / timing counters. */
pso_status pso_reset_counters(pso_handle h);

/* Destroy the handle and free its device memory.  NULL-safe. */
void pso_destroy(pso_handle h);

const char* pso_status_string(pso_status s);
const char* pso_last_error(void);
/* 1 if objective id is compiled in, else 0. */
int pso_objective_registered(int32_t objective);

/* --- NCCL plumbing for the particle-split multi-GPU path --------- *
 * NCCL is resolved at run time (dlopen of libnccl.so.2, or $PSO_NCCL_LIB), so
 * the library has no link-time NCCL dependency; inside a PyTorch process this
 * is the NCCL torch already loaded.  id is a 128-byte ncclUniqueId blob. */
pso_status pso_nccl_get_unique_id(void* id128);
pso_status pso_nccl_comm_init(void** comm, int32_t nranks, const void* id128, int32_t rank,
                              int32_t device);
pso_status pso_nccl_comm_destroy(void* comm);

/* --- NVLink peer exchange (the fused alternative to the all-gather) -------- *
 * After pso_create_ex with a communicator, every rank may switch its handle to
 * exchange gbest records by direct NVLink stores: the last CTA of each step
 * kernel writes its record (key, candidate row) into recv[t & 1][rank] of
 * every rank and releases a per-record iteration tag; the next step kernel's
 * prologue acquires the tags and merges.  No collective call per iteration.
 * Protocol (collective): each rank calls pso_p2p_handle, the 64-byte CUDA IPC
 * handles and offsets are all-gathered out of band (e.g. torch.distributed),
 * every rank calls pso_p2p_connect with the world arrays in rank order (maps
 * the peers' buffers; a failure leaves the handle on NCCL, unpoisoned), the
 * ranks agree that all connected, and then every rank calls
 * pso_p2p_enable(h, 1).  Record tags carry an epoch that pso_set_state
 * advances, so records of an earlier state never match.  A peer that stops
 * delivering makes the waiting kernels trap after 60 s (PSO_PEER_TIMEOUT_S sets
 * another limit, read at create): the handle is then poisoned (PSO_ERR_CUDA at the
 * next synchronising call) instead of the GPU hanging. */
pso_status pso_p2p_handle(pso_handle h, void* ipc_handle /* 64 bytes */, uint64_t* offset);
pso_status pso_p2p_connect(pso_handle h, const void* ipc_handles /* world x 64 bytes */,
                           const uint64_t* offsets /* world */);
/* Probe the mapped data path before enabling it (collective, two phases with a
 * host barrier between them): phase 0 stores this rank's token into its slot of
 * every rank's probe area with a system-scope release; phase 1 acquires our own
 * slots and sets *ok = 1 if every rank's token arrived (then clears them).  A
 * connected but non-working mapping is caught here rather than by the 60 s
 * trap of the first step kernel. */
pso_status pso_p2p_probe(pso_handle h, int32_t phase, int32_t* ok);
pso_status pso_p2p_enable(pso_handle h, int32_t on); /* 1: NVLink records, 0: NCCL all-gather */

/* --- Device-side primitives exposed for parity tests ---------------------- */
/* out[k] = word(tag, t, i, j0 + k) computed on the device (k < m), with the
 * library's Philox (use_curand = 0) or with curand_Philox4x32_10 (1).
 * word(tag,t,i,j) = Philox4x32-10(ctr = {j>>2, i, t, tag}, key = {seed lo, hi})[j&3]. */
pso_status pso_debug_philox(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j0,
                            int64_t m, uint32_t* out, int32_t use_curand, int32_t device);
/* Evaluate m rows (dense m x d host matrix X) on the device with the same
 * functor + CTA reduction the fused kernel uses; out receives m floats. */
pso_status pso_debug_objective(int32_t objective, const float* X, int64_t m, int32_t d,
                               float* out, int32_t device);

#ifdef __cplusplus
}
#endif
#endif /* FASTPSO_H */
