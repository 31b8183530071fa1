"""Oracle of the asynchronous particle split (NEXT-4) — TEST INFRASTRUCTURE ONLY.

P:L281: "the whole particle group is split into multiple sub-groups.  Each
sub-group is assigned to a card for optimization, and maintains its own
local-global best information.  The global information of the whole group can
be updated in an asynchronous manner."  Reading (reading 26): a
fixed one-iteration lag, so the result is deterministic for a given number of
shards.  Built only from the pinned shard primitives of the C oracle
(init_local / step_local / merge), in this order per iteration t:

  1. every shard merges the records (best strictly-improving row of each
     shard) of iteration t - 2 (iteration 0 for t < 2) into its own gbest
     (adopted only if strictly better; the lowest (f, i) among records wins);
  2. Alg. 1 body on the shard's rows with the shard's own gbest as G;
  3. the shard adopts its own candidate at once and publishes it as its
     record of iteration t.

Initialisation is synchronous (every shard starts from the global best of
iteration 0), and so is set_state at iteration t0: records then start at t0
and step t merges those of max(t - 2, t0).  The host's view after a pso_step call: each shard's gbest merged
with the records of the last two iterations.
"""
from __future__ import annotations

import numpy as np

from . import OracleSwarm


class AsyncSplitSwarm:
    def __init__(self, n, d, w, c1, c2, lo, hi, objective, seed, k, vmax=0.0, bounds=None):
        self.n, self.d, self.k = int(n), int(d), int(k)
        self.shards = []
        for r in range(self.k):
            b, e = (n * r) // k, (n * (r + 1)) // k
            self.shards.append(OracleSwarm(n, d, w, c1, c2, lo, hi, objective, seed, vmax=vmax,
                                           row_begin=b, nrows=e - b, create=False, bounds=bounds))
        recs = [s.init_local() for s in self.shards]
        for s in self.shards:  # synchronous start: everyone adopts the global best of iteration 0
            self._merge(s, recs, is_init=True)
        self.records = {0: recs}
        self.t = 0
        self.t_base = 0  # iteration of the last synchronous (re-)selection

    def _merge(self, shard, recs, is_init=False):
        has = [bool(r[0]) for r in recs]
        shard.merge(has, [r[1] for r in recs], [r[2] for r in recs],
                    np.stack([r[3] for r in recs]), is_init)

    def step(self, iters=1):
        for _ in range(int(iters)):
            t = self.t + 1
            lagged = self.records[t - 2 if t >= self.t_base + 2 else self.t_base]
            out = []
            for s in self.shards:
                self._merge(s, lagged)
                rec = s.step_local()  # strict candidate vs the shard's own gbest
                if rec[0]:
                    self._merge(s, [rec])  # adopt own candidate at once
                out.append(rec)
            self.records[t] = out
            self.records.pop(t - 3, None)
            self.t = t
        return self

    def set_state(self, states, t):
        """Restore every shard's (X, V, PB, pf) at iteration t: a synchronous
        re-selection (each shard's best pbest row, then the global minimum of
        (f, i) everywhere), after which the lag restarts from t."""
        recs = []
        for s, (X, V, PB, pf) in zip(self.shards, states):
            s.set_state(X, V, PB, pf, t=t)
            recs.append((s.nrows > 0, s.gf, s.gi, s.G.copy()))
        for s in self.shards:
            self._merge(s, recs, is_init=True)
        self.records = {int(t): recs}
        self.t = self.t_base = int(t)
        return self

    def view(self, shard=0):
        """(gf, gi, G) the host reads after a pso_step call on `shard`'s rank."""
        s = self.shards[shard]
        gf, gi = s.gf, s.gi
        best = (gf, gi, s.G.copy())
        cands = [(f, i, row) for it in (self.t - 1, self.t) if it >= self.t_base
                 for has, f, i, row in self.records.get(it, []) if has and f < gf]
        if cands:
            f, i, row = min(cands, key=lambda c: (c[0], c[1]))
            best = (f, i, row.copy())
        return best

    def state(self, shard):
        s = self.shards[shard]
        return s.X, s.V, s.PB, s.pf, s.t
