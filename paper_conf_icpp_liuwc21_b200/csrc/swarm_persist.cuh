// swarm_persist.cuh — the persistent streaming step kernel (SURVEY 8(f) NEXT-1,
// the latency path for swarms too large for the grid's shared memory but too
// small to hide a kernel boundary per iteration; C3: 10k x 1000).  Included by
// swarm_kernels.cuh inside namespace fastpso::{anon}.
//
// One cooperative launch runs a whole pso_step call.  Every CTA is a k_step_tma
// pipeline (producer / compute / finaliser warps, bulk copies through a ring of
// row stages) over a FIXED set of rows, b, b + grid, ... (no dynamic claims, no
// serpentine order), for every iteration of the call:
//
//   finaliser  per row: the k_step_tma decision and bulk stores; a row that
//              becomes the CTA's best gbest candidate is also bulk-stored into
//              cand[t & 1][b].  After its last row of iteration t it waits for
//              every store (bulk wait_group 0), tells the producer (mbarrier
//              itdone), atomicMin's its candidate key into key_acc[t & 1]
//              (ctl->key_acc / ctl->key_acc1) and arrives at a grid barrier
//              (ticket + generation, as k_gridres); then it reads the winner
//              key, pulls the winner's row from cand[t & 1][owner] into sG and
//              releases the compute warps (mbarrier gready).
//   producer   loads the rows of iteration t + 1 as soon as itdone says this
//              CTA's stores (and lazy flags) of iteration t are complete -- the
//              rows are its own, so the loads overlap the grid barrier; only G
//              waits for it.
//   compute    per iteration: wait gready, then the k_step_tma row body.
//
// Per row the arithmetic, the reduction order and the decisions are
// k_step_tma's, so the state is bitwise the streaming kernel's (tests).  The
// last arriver of the barrier of iteration t resets key_acc[(t + 1) & 1]
// (every CTA read it after the barrier of t - 1); after the last iteration a
// final ticket's last arriver writes G, key_cur, t and resets both key slots.
// Single GPU only (no exchange).

// (80 registers: four CTAs of 4 compute warps per SM, k_step_tma's C3 shape)
template <class Obj, int VPT, bool kB>
__global__ void __maxnreg__(80)
    k_step_persist(const __grid_constant__ SwarmArgs a, int iters, int stages) {
  extern __shared__ __align__(128) unsigned char dsmem[];
  const int nvec = a.nvec, d = a.d;
  const int nthr = (int)blockDim.x - 64;  // compute threads
  const int nwarps = nthr >> 5;
  const int grid = (int)gridDim.x, b = (int)blockIdx.x;
  const long long n = a.n_local;
  const int myrows = b < n ? (int)((n - b + grid - 1) / grid) : 0;  // rows b, b + grid, ...
  // the CTA's m-th row of iteration t: serpentine (a.serp) walks the CTA's rows
  // backwards on odd iterations, so an iteration starts on the rows the last
  // one wrote last (L2); rows are independent, so the order changes no bit
  const bool serp = a.serp != 0;
  auto row_of = [&](uint32_t t, int m) -> long long {
    const int mm = (serp && (t & 1u)) ? myrows - 1 - m : m;
    return b + (long long)mm * grid;
  };
  float4* sG = reinterpret_cast<float4*>(dsmem);
  float4* sB = sG + nvec;  // kB: [vlo | vhi | xlo | xhi]
  float4* ring = sB + (kB ? 4 * nvec : 0);
  __shared__ float red[kMaxStages][(kMaxThreads / 32) * 2];
  __shared__ unsigned long long full[kMaxStages], empty[kMaxStages], done[kMaxStages];
  __shared__ unsigned long long gready, itdone;
  __shared__ int sflag[kMaxStages];  // lazy pbest: the stage's row had PB == X (pb not loaded)
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    mbar_init(&gready, 1);
    mbar_init(&itdone, 1);
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&done[s], (unsigned)nwarps);
      mbar_init(&empty[s], 1);
    }
    mbar_fence_init();
  }
  __syncthreads();
  const uint32_t t0 = a.ctl->t;
  const unsigned row_bytes = (unsigned)nvec * 16u;

  if (warp == nwarps) {  // ---------------- producer
    if (lane == 0) {
      int s = 0;
      unsigned ph = 0;
      long long k = 0;  // row sequence number over the whole call
      const int pd = a.l2pf;  // L2 prefetch distance in own rows (lazy rows only, as k_step_tma)
      for (int it = 0; it < iters; ++it) {
        // this CTA's stores and lazy flags of the previous iteration are complete
        // (a CTA without rows never waits: its finaliser's phases run ahead)
        if (it > 0 && myrows > 0) mbar_wait(&itdone, (unsigned)((it - 1) & 1));
        const uint32_t t = t0 + 1u + (uint32_t)it;
        // lazy flags loaded one row ahead (their L2 latency overlaps the wait for
        // a free stage instead of delaying the copies), as in k_step_tma
        const bool lz = a.lazy_pb != 0;
        int fl_next = (lz && myrows > 0) ? (int)a.pbx[row_of(t, 0)] : 0;
        int pfl_next = (pd && lz && pd < myrows) ? (int)a.pbx[row_of(t, pd)] : 0;
        for (int m = 0; m < myrows; ++m, ++k) {
          const long long r = row_of(t, m);
          const int fl = fl_next;
          if (lz && m + 1 < myrows) fl_next = a.pbx[row_of(t, m + 1)];
          if (pd && lz && m + pd < myrows) {
            const long long r2 = row_of(t, m + pd);
            const int pfl = pfl_next;
            if (m + 1 + pd < myrows) pfl_next = a.pbx[row_of(t, m + 1 + pd)];
            if (pfl || a.l2pf_all) {
              const size_t po = (size_t)r2 * 4 * nvec;
              bulk_prefetch_l2(a.X + po, row_bytes);
              bulk_prefetch_l2(a.V + po, row_bytes);
            }
          }
          if (k >= stages) mbar_wait(&empty[s], ph ^ 1u);
          float4* st = ring + (size_t)s * 3 * nvec;
          PSO_DCHECK(r >= 0 && r < n && s < stages && stages <= kMaxStages);
          PSO_DCHECK((size_t)((const unsigned char*)(st + 3 * nvec) - dsmem) <= dyn_smem_bytes());
          sflag[s] = fl;
          mbar_expect_tx(&full[s], (fl ? 2u : 3u) * row_bytes);  // releases sflag[s] too
          bulk_g2s(st, a.X + (size_t)r * 4 * nvec, row_bytes, &full[s]);
          bulk_g2s(st + nvec, a.V + (size_t)r * 4 * nvec, row_bytes, &full[s]);
          if (!fl) bulk_g2s(st + 2 * nvec, a.PB + (size_t)r * 4 * nvec, row_bytes, &full[s]);
          if (++s == stages) {
            s = 0;
            ph ^= 1u;
          }
        }
      }
    }
    return;
  }

  if (warp == nwarps + 1) {  // ---------------- finaliser (+ the grid barrier and the G pull)
    const float4* G4 = reinterpret_cast<const float4*>(a.G);
    for (int q = lane; q < nvec; q += 32) sG[q] = G4[q];
    if (kB)
      for (int q = lane; q < 4 * nvec; q += 32) sB[q] = reinterpret_cast<const float4*>(a.bounds)[q];
    unsigned long long cur = a.ctl->key_cur;
    const unsigned gen0 = ld_acquire_u32(&a.ctl->bar_gen);  // barrier `it` completes at gen0 + it + 1
    __syncwarp();
    if (lane == 0) mbar_arrive(&gready);  // iteration 0: G of the previous call
    unsigned nimp = 0, n_pbl = 0, n_pbs = 0;
    int s = 0, prev = -1;
    unsigned ph = 0;
    for (int it = 0; it < iters; ++it) {
      const uint32_t t = t0 + 1u + (uint32_t)it;
      const int par = (int)(t & 1u);
      unsigned long long win = ~0ull;
      if (lane == 0) {
        const uint32_t inc_ord = (uint32_t)(cur >> 32);
        unsigned long long best = ~0ull;
        bool cand_pending = false;
        float* cand_row = a.cand + ((size_t)par * grid + b) * 4 * nvec;
        for (int m = 0; m < myrows; ++m) {
          const long long r = row_of(t, m);
          mbar_wait(&full[s], ph);
          const float pf_old = a.pf[r];
          const uint32_t gi = (uint32_t)(a.row_begin + r);
          mbar_wait(&done[s], ph);
          float c[Obj::kAcc];
          Obj::init(c);
          for (int w = 0; w < nwarps; ++w) {
            float bw[Obj::kAcc];
#pragma unroll
            for (int j = 0; j < Obj::kAcc; ++j) bw[j] = red[s][w * Obj::kAcc + j];
            Obj::combine(c, bw);
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
          if (f == f && ord_f32(f) < inc_ord) {  // strictly below gf (Alg. 1 line 10)
            const unsigned long long key = pack_key(f, gi);
            if (key < best) {  // x' is the row's new pbest: the CTA's candidate row
              if (cand_pending) bulk_wait_all();  // two bulk stores to one address: in order
              best = key;
              bulk_s2g(cand_row, xnew, row_bytes);
              cand_pending = true;
            }
          }
          bulk_commit();
          if (prev >= 0) {  // the previous row's stores have read their stage
            bulk_wait_read<1>();
            mbar_arrive(&empty[prev]);
          }
          prev = s;
          if (++s == stages) {
            s = 0;
            ph ^= 1u;
          }
        }
        bulk_wait_all();  // every X / V / PB / candidate row of the iteration written
        fence_proxy_async_global();
        if (prev >= 0) {  // the last stage of the iteration is free
          mbar_arrive(&empty[prev]);
          prev = -1;
        }
        mbar_arrive(&itdone);  // (release: the pf / pbx stores above) the producer may load it + 1
        unsigned long long* kacc = par ? &a.ctl->key_acc1 : &a.ctl->key_acc;
        unsigned long long* knext = par ? &a.ctl->key_acc : &a.ctl->key_acc1;
        if (best != ~0ull) atomicMin(kacc, best);
        __threadfence();
        // grid barrier (acq_rel ticket; the last arriver resets the other key
        // slot -- iteration it + 1's, read by every CTA after barrier it - 1 --
        // and releases the generation)
        const unsigned gen_done = gen0 + (unsigned)it + 1u;
        if (atom_add_acq_rel_u32(&a.ctl->bar_count, 1u) == (unsigned)grid - 1) {
          a.ctl->bar_count = 0;
          *knext = ~0ull;
          st_release_u32(&a.ctl->bar_gen, gen_done);
        } else {
          while (ld_acquire_u32(&a.ctl->bar_gen) != gen_done) {
          }
        }
        win = *(volatile unsigned long long*)kacc;
      }
      win = __shfl_sync(kFull, win, 0);
      if (win < cur) {  // strictly better than the incumbent (candidates already are)
        const long long wr = (long long)(uint32_t)win - a.row_begin;
        const int owner = (int)(wr % grid);
        PSO_DCHECK(wr >= 0 && wr < n);
        const float4* src = reinterpret_cast<const float4*>(a.cand) + ((size_t)par * grid + owner) * nvec;
        for (int q = lane; q < nvec; q += 32) sG[q] = __ldcg(src + q);
        cur = win;
      }
      __syncwarp();
      if (lane == 0 && it + 1 < iters) mbar_arrive(&gready);  // G of iteration it + 1
    }
    if (lane == 0) {
      if (nimp) atomicAdd(&a.ctl->improvements, (unsigned long long)nimp);
      if (n_pbl) atomicAdd(&a.ctl->pb_loads, (unsigned long long)n_pbl);
      if (n_pbs) atomicAdd(&a.ctl->pb_stores, (unsigned long long)n_pbs);
    }
    // final ticket: every CTA has read the last key slot; its last arriver
    // publishes the call's result (G, key_cur, t) and resets both key slots
    int last = 0;
    if (lane == 0) {
      __threadfence();
      last = atom_add_acq_rel_u32(&a.ctl->bar_count, 1u) == (unsigned)grid - 1;
      if (last) {
        a.ctl->bar_count = 0;
        a.ctl->key_acc = ~0ull;
        a.ctl->key_acc1 = ~0ull;
        a.ctl->key_cur = cur;
        a.ctl->t = t0 + (uint32_t)iters;
        a.ctl->done = 0;
        st_release_u32(&a.ctl->bar_gen, gen0 + (unsigned)iters + 1u);
      }
    }
    last = __shfl_sync(kFull, last, 0);
    if (last) {
      float4* Gout = reinterpret_cast<float4*>(a.G);
      for (int q = lane; q < nvec; q += 32) Gout[q] = sG[q];
    }
    return;
  }

  // ---------------- compute warps (k_step_tma's row body)
  const PhiloxRoundKeys& key = a.rk;
  const MoveParams mp = move_params(a);
  constexpr bool kTab = HasRowTable<Obj>::value && !Obj::kNeighbor && VPT <= 2;
  float4 rtab[VPT];
  if constexpr (kTab) {
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int q = tid + j * nthr;
      rtab[j] = q < nvec ? Obj::table4(4 * q) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
  // row-invariant Philox rounds of this thread's slots (k_step_tma's narrow rule)
  constexpr bool kSlotRng = PSO_SLOT_PHILOX && PSO_SLOT_PHILOX_NARROW && VPT <= 2 && !Obj::kNeighbor && !kB;
  PhiloxSlot ps1[VPT], ps2[VPT];
  int s = 0;
  unsigned ph = 0;
  for (int it = 0; it < iters && myrows > 0; ++it) {
    const uint32_t t = t0 + 1u + (uint32_t)it;
    const PhiloxIter pit = philox_iter(key, t);
    if constexpr (kSlotRng) {
#pragma unroll
      for (int j = 0; j < VPT; ++j) {
        const uint32_t q = (uint32_t)(tid + j * nthr);
        ps1[j] = philox_slot(key, pit, q, kTagR1);
        ps2[j] = philox_slot(key, pit, q, kTagR2);
      }
    }
    mbar_wait(&gready, (unsigned)(it & 1));  // G of this iteration is in sG
    for (int m = 0; m < myrows; ++m) {
      const long long r = row_of(t, m);
      float4* st = ring + (size_t)s * 3 * nvec;
      mbar_wait(&full[s], ph);
      const uint32_t gi = (uint32_t)(a.row_begin + r);
      // lazy pbest row (PB == X): pb is the loaded x, and x' goes to the pb slot
      // so the old x stays available for a deferred PB store
      const int fl = sflag[s];
      float4* xdst = fl ? st + 2 * nvec : st;
      float acc[Obj::kAcc];
      Obj::init(acc);
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
}
