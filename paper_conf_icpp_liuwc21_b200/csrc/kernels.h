// kernels.h — internal interface between the C ABI (api.cpp) and the CUDA
// kernels (swarm_kernels.cu, debug_kernels.cu).  Not part of the public ABI.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace fastpso {

// Per-handle control block in device memory (one cache line).
struct DevCtl {
  unsigned long long key_cur;       // incumbent gbest key: ord(gf) << 32 | gi
  unsigned long long key_acc;       // atomicMin accumulator of this iteration
  unsigned long long improvements;  // pbest improvements, summed
  unsigned int done;                // last-CTA ticket counter
  unsigned int t;                   // iterations done (low 32 bits; Philox ctr[2])
  unsigned long long row_claim;     // TMA streaming kernel, dynamic rows: rows claimed beyond the
                                    // grid's first (reset by the iteration's last CTA)
  unsigned long long key_acc1;      // persistent kernel: the atomicMin slot of odd iterations
  unsigned int bar_count, bar_gen;  // grid-resident kernel: grid barrier
  unsigned long long pb_loads;      // streaming kernels: pbest rows read from HBM
  unsigned long long pb_stores;     // streaming kernels: pbest rows written to HBM
  unsigned long long key_view;      // async: global gbest key folded for the host
  unsigned long long pad[6];
};
static_assert(sizeof(DevCtl) == 128, "DevCtl is two 64-byte blocks");

// Philox4x32-10 key schedule of the seed, precomputed on the host (round r:
// seed_lo + r 0x9E3779B9, seed_hi + r 0xBB67AE85).  Read through a reference
// to the kernel parameter, every round key is a constant-bank operand of the
// LOP3 that consumes it instead of a per-call uniform add (philox.cuh).
struct PhiloxRoundKeys {
  unsigned int k0[10], k1[10];
#ifdef __CUDACC__
  __device__ __forceinline__ unsigned int rk0(int r) const { return k0[r]; }
  __device__ __forceinline__ unsigned int rk1(int r) const { return k1[r]; }
#endif
  void set(unsigned long long seed) {
    for (int r = 0; r < 10; ++r) {
      k0[r] = (unsigned)seed + (unsigned)r * 0x9E3779B9u;
      k1[r] = (unsigned)(seed >> 32) + (unsigned)r * 0xBB67AE85u;
    }
  }
};

// Exchange record for world > 1: the local candidate key and its PB row.
// Layout: [u64 key][u64 pad][pitch floats].
__host__ __device__ inline size_t record_bytes(int pitch) { return 16 + (size_t)pitch * 4; }

struct SwarmArgs {
  float* X;   // n_local x pitch
  float* V;
  float* PB;
  float* pf;  // n_local
  float* G;   // pitch (gbest position)
  float* cand;                // grid-resident kernel: [2][grid][pitch] candidate rows
  unsigned long long* cand_key;  // grid-resident kernel: [2][grid] candidate keys (~0: none)
  const float* bounds;        // per-dimension bounds [vlo | vhi | xlo | xhi] (4 x pitch), or null
  unsigned char* pbx;         // lazy pbest: bit 0 = the row's pbest equals its x (PB not stored);
                              // bit 1 (column split) = x in the PB array, pb in X
  int lazy_pb;
  int l2pf;                   // TMA producer: L2 prefetch distance in rows of this CTA (0: off)
  int serp;                   // streaming kernels: odd iterations visit rows backwards (L2 reuse)
  int l2pf_all;               // prefetch every row (default: lazy rows only, whose stage loads 2 of 3 slots)
  int dyn_rows;               // rows / items claimed from ctl->row_claim instead of round robin:
                              // bit 0 streaming + column split, bit 1 cluster
  unsigned char* send;        // world > 1: this rank's exchange record
  const unsigned char* recv;  // exchange: [2 iteration parities][world] records after the all-gather
  DevCtl* ctl;
  long long n_local;
  long long row_begin;
  int d, nvec;                // nvec = pitch / 4
  int world;
  int rank;
  int exchange;               // 1: publish (key, row) records for the all-gather + select
  int xrecs;                  // records per iteration slot the merges read: world (all-gather,
                              // NVLink), or 1 (allreduce exchange: the reduced record)
  int p2p;                    // exchange over NVLink peer stores instead of NCCL
  int async_gbest;            // NEXT-4: merge peers' records with a one-iteration lag
  float* G_view;              // async: the host's global gbest view (pitch floats)
  unsigned epoch;             // p2p: record tags are (epoch << 32 | t); set_state starts an epoch
  unsigned t_base;            // async: iteration of the last create/set_state (records start there)
  unsigned char* const* peers;  // p2p: device array, world pointers to every rank's recv
  unsigned long long peer_timeout_ns;  // p2p: a peer record not arriving within this traps the
                                       // kernel (a dead rank poisons the handle instead of hanging)
  unsigned long long probe_off; // p2p: offset from a recv base to the connect probe slots (world u64)
  // Column split (NEXT-3, "tile matrix"): this rank holds float4 columns
  // [col_q0, col_q0 + nvec) of every row (n_local = n); X, V, PB, G, bounds are
  // that block (pitch 4 nvec).  recv = [2][world] u64 tags, then the partials
  // [2 parities][n][col_nbt] float4 {acc0, acc1, first x', last x'}.
  int colsplit;
  int col_q0;       // first global float4 of the block
  int nvec_glob;    // float4 of a full row
  int col_chunk;    // float4 per local tile (a row of the block is col_nb tiles)
  int col_nb;       // local tiles per row
  int col_bbase;    // index of this rank's first tile among all ranks' tiles
  int col_nbt;      // tiles per row over all ranks
  float w, c1, c2, lo, hi, vmax;
  unsigned int seed_lo, seed_hi;
  PhiloxRoundKeys rk;  // the same seed's Philox key schedule
};

// Column split geometry (host plan and decide kernel).  The tiling depends on
// d only, never on the world size: rows of nvec = ceil(d / 4) float4 are cut
// into tiles of T = clamp(ceil(nvec / 8), 32, 512) float4 (the last one
// ragged), and rank r of `world` owns tiles [floor(nt r / world),
// floor(nt (r+1) / world)).  The partial of a tile and the combine order over
// tiles are therefore the same for every world size, so fitness, decisions
// and state are bitwise independent of it.
constexpr int kColTileMax = 512, kColTileMin = 32;
__host__ __device__ inline int col_tile(int nvec) {
  int t = (nvec + 7) / 8;  // >= 8 tiles (8 ranks) from 256 float4 up, 8 KB tiles for wide rows
  t = t < kColTileMin ? kColTileMin : (t > kColTileMax ? kColTileMax : t);
  return t < nvec ? t : nvec;
}
__host__ __device__ inline int col_ntiles(int nvec) {
  const int t = col_tile(nvec);
  return (nvec + t - 1) / t;
}
__host__ __device__ inline void col_rank_tiles(int ntiles, int world, int r, int* t0, int* nt) {
  const long long b = (long long)ntiles * r / world, e = (long long)ntiles * (r + 1) / world;
  *t0 = (int)b;
  *nt = (int)(e - b);
}
__host__ __device__ inline size_t col_tag_bytes(int world) {
  return ((size_t)2 * world * 8 + 255) / 256 * 256;
}

struct LaunchCfg {
  int vpt = 1;        // float4 per compute thread per row
  int compute = 32;   // compute threads per CTA (one row per CTA at a time)
  int threads = 32;   // CTA size (compute + 32 producer threads for the TMA pipeline)
  int grid = 1;       // persistent grid
  int ctas_per_sm = 1;
  int tma = 0;        // 1: warp-specialised bulk-copy (TMA) pipeline; 0: register streaming
  int wide = 0;       // TMA pipeline: the 512-compute-thread instantiation
  int stages = 0;     // TMA pipeline depth (rows in flight per CTA)
  size_t smem = 0;    // dynamic shared memory bytes of the step kernel
  int resident = 0;   // 1: tiny swarm, whole pso_step in one single-CTA launch
  int gridres = 0;    // 1: swarm held in the grid's shared memory (cooperative launch)
  int persist = 0;    // 1: persistent streaming kernel, a whole pso_step per cooperative launch
  int persist_grid = 0;
  int cluster = 0;    // > 0: rows split across a thread-block cluster of this many CTAs
  int chunk = 0;      // float4 per CTA block in the cluster path
  int init_threads = 0;
  int init_vpt = 1;
  int gridres_grid = 0;
  int gridres_rows = 0;     // max rows per CTA
  size_t gridres_smem = 0;
  int resident_threads = 0;
  size_t resident_smem = 0;
  size_t init_smem = 0;
  int bounds = 0;     // kernels instantiated with per-dimension bounds
  int pdl = 1;        // step kernels: programmatic dependent launch (PSO_PDL=0 disables)
  int colsplit = 0;   // column split: k_col_step + k_col_decide per iteration
  int col_grid = 0, col_stages = 0, col_decide_grid = 0;
  size_t col_smem = 0, col_decide_smem = 0;
};

// Tuning overrides (0 / -1 = automatic): PSO_VPT, PSO_KERNEL=reg|tma, PSO_STAGES, PSO_CTAS.
struct PlanHints {
  int vpt = 0;
  int kernel = -1;  // -1 auto, 0 register, 1 tma
  int stages = 0;
  int ctas = 0;     // max CTAs per SM for the TMA pipeline (0: auto = 2)
  bool allow_resident = false;  // single-GPU tiny swarms (PSO_RESIDENT=0 disables)
  int persist = -1;             // persistent streaming kernel: -1 auto, 0 off, 1 on (PSO_PERSIST)
  bool bounds = false;          // per-dimension bounds tables are in use
  int cluster = 0;              // force the cluster path with this many CTAs (PSO_CLUSTER)
};

// Kernel entry points of one objective functor: [VPT index 1,2,4,8][per-dim bounds].
struct KernelTable {
  bool neighbor;
  const void* step_reg[4][2];
  const void* step_tma[4][2];
  const void* step_tma_w[4][2];  // 512 compute threads, one CTA per SM (VPT 2 and 4 only)
  const void* gridres[4][2];
  const void* step_cluster[4][2];
  const void* persist[4][2];     // persistent streaming kernel (swarm_persist.cuh)
  const void* resident[2];
  const void* init[4];
  const void* eval[4];
  const void* col_step[2];  // [per-dim bounds]
  const void* col_decide;
};
// The table of a registered objective id, or null (obj_*.cu).
const KernelTable* kernel_table(int objective);

bool objective_registered(int objective);
// Choose the CTA shape for d and size the persistent grid for n_local rows.
cudaError_t plan_launch(int objective, int d, long long n_local, int sm_count, const PlanHints& h,
                        LaunchCfg* cfg);
cudaError_t launch_init(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s);
cudaError_t launch_step(int objective, const SwarmArgs& a, const LaunchCfg& c, cudaStream_t s);
cudaError_t launch_resident(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                            cudaStream_t s);
cudaError_t launch_gridres(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                           cudaStream_t s);
cudaError_t launch_persist(int objective, const SwarmArgs& a, const LaunchCfg& c, int iters,
                           cudaStream_t s);
// Column split (NEXT-3): tile plan for this rank's block, and the two kernels
// of an iteration (init = 1: Alg. 1 lines 1-3 instead of the move).
cudaError_t plan_colsplit(int objective, int tile, int tiles_local, long long n, int sm_count,
                          bool bounds, LaunchCfg* cfg);
cudaError_t launch_col_step(int objective, const SwarmArgs& a, const LaunchCfg& c, int init,
                            cudaStream_t s);
cudaError_t launch_col_decide(int objective, const SwarmArgs& a, const LaunchCfg& c, int init,
                              cudaStream_t s);
cudaError_t launch_rebest(const SwarmArgs& a, unsigned t, cudaStream_t s);
// Fold the records of iteration t (and, asynchronous, of t - 1) for the host;
// into_local: also into the kernels' incumbent (create / set_state).
cudaError_t launch_select(const SwarmArgs& a, unsigned t, bool into_local, cudaStream_t s);
// A rank without particles: its share of iteration t of the exchange (merge the
// records of t - 1 if `merge`, publish a "no candidate" record of t).
cudaError_t launch_empty_step(const SwarmArgs& a, unsigned t, bool merge, cudaStream_t s);
// Allreduce exchange: after the allreduce-min of the keys into record 0 of the
// current slot, the owner of the winning key writes its candidate row there and
// every other rank zeros it (the allreduce-sum that follows broadcasts the bits).
cudaError_t launch_owner_row(const SwarmArgs& a, cudaStream_t s);
// NVLink connect probe: phase 0 stores this rank's token into every peer's probe
// slot; phase 1 (after a host barrier) checks that every peer's token arrived in
// ours (*ok_dev = 1) and clears the slots.
cudaError_t launch_p2p_probe(const SwarmArgs& a, int phase, int* ok_dev, cudaStream_t s);
// lazy pbest: copy X -> PB for flagged rows and clear the flags (host reads)
cudaError_t launch_materialize_pb(const SwarmArgs& a, cudaStream_t s);

cudaError_t debug_philox(unsigned long long seed, unsigned tag, unsigned t, unsigned i,
                         unsigned j0, long long m, unsigned* out_dev, int use_curand,
                         cudaStream_t s);
cudaError_t debug_objective(int objective, const float* X_dev, long long m, int d, int pitch,
                            float* out_dev, int sm_count, cudaStream_t s);

}  // namespace fastpso
