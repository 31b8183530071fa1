// swarm_colsplit.cuh — the column split (the
// paper's second multi-GPU approach: "tile the matrix").  Included by
// swarm_kernels.cuh inside namespace fastpso::{anon}.
//
// Each rank holds a block of whole tiles of EVERY row (kernels.h col_tile);
// one iteration is two kernels:
//
//   k_col_step    the Eq. 1 move of the rank's tiles (a tile = up to kColTile
//                 float4 of one row), streamed through the same warp-specialised
//                 TMA ring as k_step_tma (producer warp: bulk copies of x, v, pb
//                 and the G tile; compute warps: Philox + move + the functor's
//                 map over the tile; finaliser warp: warp partials -> the tile's
//                 partial {acc0, acc1, first x', last x'}, bulk stores of x', v').
//                 The tile partial is stored into the partial table of every
//                 rank (own memory, and the peers' over NVLink, CUDA-IPC-mapped);
//                 the last CTA then releases this rank's tag of iteration t.
//   k_col_decide  acquires every rank's tag, combines a row's tile partials in
//                 tile order (plus the neighbour terms x_j, x_{j+1} across tile
//                 borders), finalises f, and takes the pbest decision (Alg. 1
//                 lines 7-9) and the gbest argmin (lines 10-12) -- every rank
//                 computes the same bits from the same table, so the decisions
//                 agree without another exchange.  The last CTA copies the
//                 winner's x (this rank's block) into G.
//
// The pbest copy cannot wait for the decision (x' is stored before f is
// known), so a row's position and pbest live in two slots, the X and the PB
// array, and pbx[r] records where (round 3 of the design):
//   bit 0 (lazy)  the row improved in the last decision: its pbest IS its
//                 position (one slot holds both, the other is stale);
//   bit 1 (swap)  the position lives in the PB array (and a non-lazy row's
//                 pbest in the X array).
// A non-lazy row reads x and pb and stores x' over x (same slot).  A lazy row
// reads only x (= pb) and stores x' into the OTHER slot, so the old x stays
// in place as the pbest should the row not improve -- no copy, ever:
//   new swap bit = lazy ? !swap : swap,   new lazy bit = improved.
// Bytes per element: 16 (x, v in and out) + 4 for a row that did not improve
// in the last decision (its pb read).  k_materialize_pb restores the plain
// layout (X = x, PB = pb) before the host reads whole matrices.
//
// Init (init = 1, Alg. 1 lines 1-3): the producer loads nothing; the compute
// warps draw x0, v0 (Philox X0 / V0 at the global column), the finaliser stores
// X, V and PB = x0, and k_col_decide sets pf = f (NaN -> +inf) and selects the
// global best from scratch.

template <class Obj>
__device__ __forceinline__ float4* col_parts(unsigned char* region, const SwarmArgs& a, int par) {
  return reinterpret_cast<float4*>(region + col_tag_bytes(a.world)) +
         (size_t)par * (size_t)a.n_local * (size_t)a.col_nbt;
}

constexpr int kColCompute = 256;  // compute threads of k_col_step (+ producer + finaliser warps)
static_assert(kColTileMax <= 2 * kColCompute, "k_col_step: at most 2 float4 of a tile per thread");

template <class Obj, bool kB>
__global__ void __launch_bounds__(kColCompute + 64, 2)
    k_col_step(const __grid_constant__ SwarmArgs a, int init, int stages) {
  static_assert(Obj::kAcc <= 2, "the tile partial carries two accumulators");
  extern __shared__ __align__(128) unsigned char dsmem[];
  constexpr int nthr = kColCompute, nwarps = nthr / 32;
  // Shared memory: [G cache: 2 slots x gper tiles][ring: stages x {x, v, pb}].
  // Items are visited tile-major, so a CTA's consecutive items mostly share
  // their column tile: the G tile (and the bounds tiles) is loaded into one of
  // two cache slots only when the tile changes, and the stages hold just the
  // row arrays -- 4 stages of 24 KB instead of 3 of 32 KB at 512-float4 tiles.
  constexpr int per = 3;            // stage arrays: x, v, pb
  constexpr int gper = kB ? 5 : 1;  // cache slot arrays: g [, vlo, vhi, xlo, xhi]
  const int chunk = a.col_chunk, nb = a.col_nb, nvl = a.nvec, d = a.d;
  float4* gcache = reinterpret_cast<float4*>(dsmem);
  float4* ring = gcache + 2 * gper * chunk;
  __shared__ float red[kMaxStages][nwarps * 2];
  __shared__ unsigned long long full[kMaxStages], empty[kMaxStages], done[kMaxStages];
  __shared__ int sflag[kMaxStages];
  __shared__ long long s_r[kMaxStages];  // the stage's item: row (-1: no more items) ...
  __shared__ int s_b[kMaxStages];        // ... and tile
  __shared__ int s_g[kMaxStages];        // ... and the G cache slot holding the tile
  // the tile's first and last x' for the neighbour terms across tiles, handed to
  // the finaliser by the arriving lanes themselves (ordered by their own release)
  __shared__ float s_edge[kMaxStages][2];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&done[s], (unsigned)nwarps);
      mbar_init(&empty[s], 1);
    }
    mbar_fence_init();
  }
  __syncthreads();
  pdl_wait_and_release();  // the previous iteration's decisions, G and t are visible
  const uint32_t t = init ? 0u : a.ctl->t + 1u;
  const long long items = a.n_local * (long long)nb;

  if (warp == nwarps) {  // ---------------- producer
    if (lane == 0) {
      int s = 0;
      unsigned ph = 0;
      long long i = 0;
      // Item schedule: tile-major (item k = tile k / n, row k mod n), round
      // robin or (a.dyn_rows) the first item is blockIdx.x and every further
      // one is claimed from ctl->row_claim two items ahead, each claim's value
      // consumed before the sentinel (the last CTA resets the counter).  The
      // producer passes the item's (row, tile, cache slot) with the stage.
      unsigned long long* claim_ctr = &a.ctl->row_claim;
      const bool dyn = (a.dyn_rows & 1) != 0;
      const long long n = a.n_local;
      long long k = blockIdx.x;
      long long k_next =
          k >= items ? items : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + gridDim.x : k + gridDim.x);
      // the lazy-pbest flag of the next item is loaded one item ahead, so its L2
      // latency overlaps the wait for a free stage instead of delaying the copies
      int fl_next = (!init && k < items) ? a.pbx[k % n] : 0;
      // G cache: the tile each slot holds (-1: none) and the last item using it
      int g_tile0 = -1, g_tile1 = -1;
      long long g_last0 = -1, g_last1 = -1;
      for (; k < items; ++i) {
        const int b = (int)(k / n);
        const long long r = k - (long long)b * n;
        const int q0 = b * chunk;
        const int cnt = min(chunk, nvl - q0);
        const unsigned bytes = (unsigned)cnt * 16u;
        const int fl = fl_next;
        const long long k_nn = k_next >= items ? items
                               : (dyn ? (long long)atomicAdd(claim_ctr, 1ull) + gridDim.x
                                      : k_next + gridDim.x);
        if (!init && k_next < items) fl_next = a.pbx[k_next % n];
        k = k_next;
        k_next = k_nn;
        if (i >= stages) mbar_wait(&empty[s], ph ^ 1u);
        float4* st = ring + (size_t)s * per * chunk;
        PSO_DCHECK(r >= 0 && r < n && b >= 0 && b < nb && cnt >= 1 && cnt <= chunk && s < stages);
        PSO_DCHECK((size_t)((const unsigned char*)(st + per * chunk) - dsmem) <= dyn_smem_bytes());
        PSO_DCHECK((size_t)q0 + cnt <= (size_t)nvl && stages <= kMaxStages);
        s_r[s] = r;
        s_b[s] = b;
        if (init) {
          sflag[s] = 0;
          s_g[s] = 0;
          mbar_arrive(&full[s]);
        } else {
          int gs = g_tile0 == b ? 0 : g_tile1 == b ? 1 : -1;
          const bool load_g = gs < 0;
          if (load_g) {  // the least recently used slot, once no stage in flight reads it
            gs = g_last0 <= g_last1 ? 0 : 1;
            // (stages are released in item order, and the LRU slot's last item is
            // at most i - 2, whose release needs only items up to i - 1)
            const long long m = gs ? g_last1 : g_last0;
            if (m >= 0 && m > i - stages) mbar_wait(&empty[m % stages], (unsigned)((m / stages) & 1));
            if (gs) g_tile1 = b; else g_tile0 = b;
          }
          if (gs) g_last1 = i; else g_last0 = i;
          PSO_DCHECK(gs == 0 || gs == 1);
          PSO_DCHECK((gs ? g_tile1 : g_tile0) == b);
          s_g[s] = gs;
          sflag[s] = fl;
          const bool lazy = (fl & 1) != 0;
          mbar_expect_tx(&full[s], bytes * ((lazy ? 2u : 3u) + (load_g ? (unsigned)gper : 0u)));
          const size_t off = ((size_t)r * nvl + q0) * 4;
          const float* xs = (fl & 2) ? a.PB : a.X;  // the slot of the position
          const float* ps = (fl & 2) ? a.X : a.PB;  // ... and of a non-lazy pbest
          bulk_g2s(st, xs + off, bytes, &full[s]);
          bulk_g2s(st + chunk, a.V + off, bytes, &full[s]);
          if (!lazy) bulk_g2s(st + 2 * chunk, ps + off, bytes, &full[s]);
          if (load_g) {
            float4* gc = gcache + (size_t)gs * gper * chunk;
            bulk_g2s(gc, a.G + (size_t)q0 * 4, bytes, &full[s]);
            if (kB)
              for (int m = 0; m < 4; ++m)
                bulk_g2s(gc + (1 + m) * chunk, a.bounds + ((size_t)m * nvl + q0) * 4, bytes, &full[s]);
          }
        }
        if (++s == stages) {
          s = 0;
          ph ^= 1u;
        }
      }
      // sentinel: the compute warps and the finaliser stop at a stage without an item
      if (i >= stages) mbar_wait(&empty[s], ph ^ 1u);
      s_r[s] = -1;
      mbar_arrive(&full[s]);
    }
    return;
  }

  if (warp == nwarps + 1) {  // ---------------- finaliser
    if (lane == 0) {
      const int par = (int)(t & 1u);
      // byte offset of this iteration's partial table within every rank's region
      const size_t parts_off =  // = col_parts(region, a, par) - region
          col_tag_bytes(a.world) + (size_t)par * (size_t)a.n_local * (size_t)a.col_nbt * sizeof(float4);
      unsigned n_pbl = 0;
      int s = 0, prev = -1;
      unsigned ph = 0;
      for (;;) {
        mbar_wait(&full[s], ph);
        const long long r = s_r[s];
        if (r < 0) break;
        const int b = s_b[s];
        const int q0 = b * chunk;
        const int cnt = min(chunk, nvl - q0);
        const unsigned bytes = (unsigned)cnt * 16u;
        mbar_wait(&done[s], ph);
        float c[Obj::kAcc];
        Obj::init(c);
        for (int w = 0; w < nwarps; ++w) {
          float bw[Obj::kAcc];
#pragma unroll
          for (int j = 0; j < Obj::kAcc; ++j) bw[j] = red[s][w * Obj::kAcc + j];
          Obj::combine(c, bw);
        }
        const float4* st = ring + (size_t)s * per * chunk;
        const int fl = sflag[s];
        const float4* xnew = st;  // the compute warps put x' over x
        const float4 msg = make_float4(c[0], Obj::kAcc > 1 ? c[Obj::kAcc - 1] : 0.f,
                                       Obj::kNeighbor ? s_edge[s][0] : 0.f,
                                       Obj::kNeighbor ? s_edge[s][1] : 0.f);
        const size_t pidx = (size_t)r * a.col_nbt + (size_t)(a.col_bbase + b);
        if (a.world > 1) {
          for (int q = 0; q < a.world; ++q) reinterpret_cast<float4*>(a.peers[q] + parts_off)[pidx] = msg;
        } else {
          reinterpret_cast<float4*>(const_cast<unsigned char*>(a.recv) + parts_off)[pidx] = msg;
        }
        const size_t off = ((size_t)r * nvl + q0) * 4;
        // x' over x (non-lazy row), or into the other slot (lazy row: the old x
        // stays as the pbest until the decision says otherwise)
        const bool to_pb = ((fl >> 1) ^ (fl & 1)) != 0;
        bulk_s2g((to_pb ? a.PB : a.X) + off, xnew, bytes);
        bulk_s2g(a.V + off, st + chunk, bytes);
        if (init) bulk_s2g(a.PB + off, xnew, bytes);  // PB = x0
        if (b == 0 && !init) n_pbl += (fl & 1) ? 0u : 1u;  // per row: PB read
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
      if (n_pbl) atomicAdd(&a.ctl->pb_loads, (unsigned long long)n_pbl);
      __threadfence_system();  // this CTA's partials (local and peer stores) before the ticket
      if (atomicAdd(&a.ctl->done, 1u) == gridDim.x - 1) {
        __threadfence_system();
        a.ctl->done = 0;
        a.ctl->row_claim = 0;  // every CTA's claims are done (see the producer)
        if (a.world > 1) {
          const unsigned long long tag = ((unsigned long long)a.epoch << 32) | t;
          for (int q = 0; q < a.world; ++q)
            st_release_sys_u64(a.peers[q] + ((size_t)par * a.world + a.rank) * 8, tag);
        }
      }
    }
    return;
  }

  // ---------------- compute warps
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  const float4* B4 = reinterpret_cast<const float4*>(a.bounds);
  // Row-invariant Philox rounds of this thread's two slots (k_step_tma's
  // PhiloxSlot, the same draws bit for bit): with items visited tile-major a
  // CTA's consecutive items mostly share their tile, so they are recomputed
  // only when the tile changes
  constexpr bool kSlotRng = PSO_SLOT_PHILOX && !Obj::kNeighbor && !kB;
  // likewise the functor's per-dimension factors (Griewank's 1/sqrt(k): table4 /
  // map4r, the same bits as map4)
  constexpr bool kTab = HasRowTable<Obj>::value && !Obj::kNeighbor;
  const PhiloxIter pit = philox_iter(key, t);
  PhiloxSlot ps1[2], ps2[2];
  float4 rtab[2];
  int slot_b = -1;
  int s = 0;
  unsigned ph = 0;
  for (;;) {
    float4* st = ring + (size_t)s * per * chunk;
    mbar_wait(&full[s], ph);
    const long long r = s_r[s];
    if (r < 0) break;
    const int q0 = s_b[s] * chunk;
    if constexpr (kSlotRng || kTab) {
      if (!init && s_b[s] != slot_b) {
        slot_b = s_b[s];
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const uint32_t qg = (uint32_t)(a.col_q0 + q0 + tid + j * nthr);
          if constexpr (kSlotRng) {
            ps1[j] = philox_slot(key, pit, qg, kTagR1);
            ps2[j] = philox_slot(key, pit, qg, kTagR2);
          }
          if constexpr (kTab)
            rtab[j] = (int)qg < a.nvec_glob ? Obj::table4(4 * (int)qg) : make_float4(0.f, 0.f, 0.f, 0.f);
        }
      }
    }
    const int cnt = min(chunk, nvl - q0);
    const uint32_t gi = (uint32_t)(a.row_begin + r);
    const int fl = sflag[s] & 1;  // lazy row: pb = x (its pb slot is not loaded)
    // x' over x: the old x of a lazy row stays in HBM (the other slot)
    float4* xdst = st;
    const float4* gc = gcache + (size_t)s_g[s] * gper * chunk;
    float acc[Obj::kAcc];
    Obj::init(acc);
    float e_first = 0.f, e_last = 0.f;  // x' of the tile's first / last float4 (owners only)
    // a tile is at most 2 float4 per compute thread: two unrolled, independent
    // slots (thread-sequential order over ql = tid, tid + nthr, as before); the
    // init and step bodies are separate loops so neither carries the other's
    // registers
    if (init) {
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int ql = tid + j * nthr;
        if (ql < cnt) {
          const int qg = a.col_q0 + q0 + ql;  // global float4: Philox counter, functor index
          float4 x, v;
          init_float4_at(a, key, gi, qg, B4, nvl, q0 + ql, x, v);
          if constexpr (Obj::kNeighbor) {
            if (ql == 0) e_first = x.x;
            if (ql == cnt - 1) e_last = x.w;
          }
          xdst[ql] = x;
          st[chunk + ql] = v;
          if constexpr (!Obj::kNeighbor) map4<Obj>(acc, x, 0.f, 4 * qg, d);
        }
      }
    } else {
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int ql = tid + j * nthr;
        if (ql < cnt) {
          const int qg = a.col_q0 + q0 + ql;
          float4 x = st[ql], v = st[chunk + ql];
          const float4 g = gc[ql];
          if constexpr (kSlotRng)
            move4_draw_slot<kB>(mp, key, pit, ps1[j], ps2[j], gi, fl, x, v, st + 2 * chunk + ql, g,
                                gc + chunk, chunk, ql);
          else
            move4_draw<kB>(mp, key, t, gi, (uint32_t)qg, fl, x, v, st + 2 * chunk + ql, g, gc + chunk,
                           chunk, ql);
          if ((d & 3) && qg == a.nvec_glob - 1) {
            const int jj = 4 * qg;
            if (jj + 1 >= d) x.y = v.y = 0.f;
            if (jj + 2 >= d) x.z = v.z = 0.f;
            if (jj + 3 >= d) x.w = v.w = 0.f;
          }
          if constexpr (Obj::kNeighbor) {
            if (ql == 0) e_first = x.x;
            if (ql == cnt - 1) e_last = x.w;
          }
          xdst[ql] = x;
          st[chunk + ql] = v;
          if constexpr (kTab)
            Obj::map4r(acc, x, d, rtab[j]);
          else if constexpr (!Obj::kNeighbor)
            map4<Obj>(acc, x, 0.f, 4 * qg, d);
        }
      }
    }
    if constexpr (Obj::kNeighbor) {
      team_sync(nthr);  // every x' of the tile is in the stage
      for (int ql = tid; ql < cnt; ql += nthr) {
        const int qg = a.col_q0 + q0 + ql;
        const float4 x = xdst[ql];
        if (ql + 1 < cnt) {
          map4<Obj>(acc, x, xdst[ql + 1].x, 4 * qg, d);
        } else if (qg == a.nvec_glob - 1) {
          map4<Obj>(acc, x, 0.f, 4 * qg, d);  // the row's last float4
        } else {  // x_{j+1} of the tile's last dim is in the next tile: k_col_decide adds it
          Obj::map(acc, x.x, x.y, 4 * qg, d);
          Obj::map(acc, x.y, x.z, 4 * qg + 1, d);
          Obj::map(acc, x.z, x.w, 4 * qg + 2, d);
        }
      }
    }
    warp_combine<Obj>(acc);
    if constexpr (Obj::kNeighbor) {  // only neighbour functors need the tile's edge x'
      // ql = 0 is thread 0 (lane 0 of warp 0); ql = cnt - 1 (< 2 nthr) is thread
      // (cnt - 1) mod nthr
      const int lt = cnt - 1 >= nthr ? cnt - 1 - nthr : cnt - 1;
      const float el = __shfl_sync(kFull, e_last, lt & 31);
      if (lane == 0 && warp == (lt >> 5)) s_edge[s][1] = el;
      if (tid == 0) s_edge[s][0] = e_first;
    }
    if (lane == 0) {
#pragma unroll
      for (int j = 0; j < Obj::kAcc; ++j) red[s][warp * Obj::kAcc + j] = acc[j];
    }
    fence_proxy_async_shared();  // x', v' visible to the finaliser's bulk stores
    __syncwarp();
    if (lane == 0) mbar_arrive(&done[s]);
    if (++s == stages) {
      s = 0;
      ph ^= 1u;
    }
  }
}

// One warp per row.
constexpr int kColDecideThreads = 512;
template <class Obj>
__global__ void __launch_bounds__(kColDecideThreads) k_col_decide(const __grid_constant__ SwarmArgs a, int init) {
  __shared__ unsigned long long s_best[kColDecideThreads / 32];
  __shared__ unsigned s_nimp[kColDecideThreads / 32];
  __shared__ int s_last;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  pdl_wait_and_release();  // k_col_step's partials and flags are visible
  const uint32_t t = init ? 0u : a.ctl->t + 1u;
  const int par = (int)(t & 1u);
  const int nbt = a.col_nbt;
  if (a.world > 1 && tid == 0) {  // every rank's tiles of iteration t have landed
    const unsigned long long want = ((unsigned long long)a.epoch << 32) | t;
    const unsigned long long t0 = globaltimer_ns();
    for (int q = 0; q < a.world; ++q) {
      const void* tag = a.recv + ((size_t)par * a.world + q) * 8;
      while (ld_acquire_sys_u64(tag) != want) {
        __nanosleep(64);
        if (globaltimer_ns() - t0 > a.peer_timeout_ns) __trap();
      }
    }
  }
  __syncthreads();
  const float4* P = col_parts<Obj>(const_cast<unsigned char*>(a.recv), a, par);
  const uint32_t inc_ord = (uint32_t)(a.ctl->key_cur >> 32);
  unsigned long long best = ~0ull;
  unsigned nimp = 0;
  const long long wpc = blockDim.x >> 5;
  for (long long r = blockIdx.x * wpc + warp; r < a.n_local; r += (long long)gridDim.x * wpc) {
    const float4* Pr = P + (size_t)r * nbt;
    const float pf_old = (lane == 0 && !init) ? a.pf[r] : 0.f;  // in flight with the partials
    const int fo = (lane == 0 && !init) ? a.pbx[r] : 0;
    float c[Obj::kAcc];
    Obj::init(c);
    for (int bt = lane; bt < nbt; bt += 32) {
      const float4 p = __ldcg(Pr + bt);
      const float pa[2] = {p.x, p.y};
      Obj::combine(c, pa);
      if (Obj::kNeighbor && bt + 1 < nbt) {  // x_j, x_{j+1} across the tile border
        float bterm[Obj::kAcc];
        Obj::init(bterm);
        Obj::map(bterm, p.w, __ldcg(Pr + bt + 1).z, 4 * (bt + 1) * a.col_chunk - 1, a.d);
        Obj::combine(c, bterm);
      }
    }
    warp_combine<Obj>(c);  // xor butterfly: every lane holds the same bits
    if (lane == 0) {
      const float f = Obj::finalize(c, a.d);
      const uint32_t gi = (uint32_t)(a.row_begin + r);
      float val = f;
      if (init) {
        val = (f != f) ? __int_as_float(0x7f800000) : f;  // reading 11: NaN -> +inf
        a.pf[r] = val;
        a.pbx[r] = 0;  // PB was stored (= x0)
      } else {
        const bool imp = f < pf_old;  // strict; NaN never improves
        if (imp) {
          a.pf[r] = f;
          ++nimp;
        }
        // x' went to the other slot iff the row was lazy (see k_col_step)
        const int sw = (fo >> 1) ^ (fo & 1);
        a.pbx[r] = (unsigned char)((sw << 1) | (imp ? 1 : 0));
      }
      if (val == val && ord_f32(val) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
        const unsigned long long key = pack_key(val, gi);
        best = key < best ? key : best;
      }
    }
  }
  if (lane == 0) {
    s_best[warp] = best;
    s_nimp[warp] = nimp;
  }
  __syncthreads();
  if (tid == 0) {
    for (int w = 1; w < (int)wpc; ++w) {
      best = s_best[w] < best ? s_best[w] : best;
      nimp += s_nimp[w];
    }
    if (best != ~0ull) atomicMin(&a.ctl->key_acc, best);
    if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
    __threadfence();
    s_last = (atomicAdd(&a.ctl->done, 1u) == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (!s_last) return;
  // last CTA: the winner's x' is its pbest (it improved); copy this rank's block
  if (tid == 0) {
    __threadfence();
    s_best[0] = *(volatile unsigned long long*)&a.ctl->key_acc;
    s_best[1] = a.ctl->key_cur;
    s_nimp[0] = s_best[0] < s_best[1]  // the winner's slot (its decision is visible: ticket order)
                    ? *(volatile unsigned char*)&a.pbx[(long long)(uint32_t)s_best[0] - a.row_begin]
                    : 0u;
  }
  __syncthreads();
  const unsigned long long acc = s_best[0], cur = s_best[1];
  PSO_DCHECK(acc >= cur || ((long long)(uint32_t)acc >= a.row_begin &&
                            (long long)(uint32_t)acc - a.row_begin < a.n_local));
  if (acc < cur) {  // the block is up to 1 MB: 8 independent loads in flight per thread
    const float4* x = reinterpret_cast<const float4*>((s_nimp[0] & 2u) ? a.PB : a.X) +
                      ((long long)(uint32_t)acc - a.row_begin) * a.nvec;
    float4* G4 = reinterpret_cast<float4*>(a.G);
    const int nt = blockDim.x;
    for (int q0 = tid; q0 < a.nvec; q0 += 8 * nt) {
      float4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int q = q0 + u * nt;
        if (q < a.nvec) v[u] = __ldcg(x + q);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int q = q0 + u * nt;
        if (q < a.nvec) G4[q] = v[u];
      }
    }
  }
  __syncthreads();
  if (tid == 0) {
    if (acc < cur) a.ctl->key_cur = acc;
    a.ctl->key_acc = ~0ull;
    a.ctl->t = t;
    a.ctl->done = 0;
  }
}
