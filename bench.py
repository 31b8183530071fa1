#!/usr/bin/env python
"""FastPSO hot-path benchmark (BASELINE.json metric: particle-dim updates/sec and
% of HBM roofline at 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NS|C1..C5|W16K|W64K|W256K|NS_R8|...]
    python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N ...
    python bench.py --impl reference ...   # the CPU oracle on a bounded sample

A "step" is one PSO iteration over the whole swarm: the fused kernel (move,
evaluate, pbest, gbest); for N > 1 the same kernel also stores the rank's gbest
record into every peer over NVLink and merges the peers' records of the
previous iteration (PSO_EXCHANGE=nccl: an NCCL all-gather instead).  Default workload: the north_star swarm, Rastrigin 100,000
particles x 2,000 dims (2.4 GB of fp32 state, larger than the 126 MB L2, so no
L2 flush is needed between steps).  N > 1 splits the same swarm by particles
(strong scaling).  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import OBJ_NAMES, WORKLOADS  # noqa: E402

METRIC = "particle-dim updates/sec and % of HBM roofline at 1/2/4/8 B200"
UNIT = "particle-dim updates/s"
L2_BYTES = 126 * 2**20
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json
SPEC_HBM_GBS = 8000.0      # B200 data-sheet HBM3e bandwidth (north_star's "~8 TB/s"), context only


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--workload", default="NS", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="fastpso", choices=["fastpso", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0,
                    help="CPU budget of the cpu_baseline oracle sample")
    ap.add_argument("--ref-seconds", type=float, default=150.0,
                    help="CPU budget of the whole --impl reference run (warm-up + timed steps)")
    return ap.parse_args()


def hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as fh:
            return float(json.load(fh)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def _path_name(info) -> str:
    if info["column_split"]:
        return "column-split (%d tiles per row)" % info["col_tiles"]
    if info["cluster"]:
        return "cluster (%d CTAs per row)" % info["cluster"]
    return ["streaming", "cta-resident", "grid-resident", "persistent-streaming"][info["resident"]]


def ncu_traffic(workload_name):
    """(DRAM bytes per launch of the step kernel, where that number comes from):
    the committed ncu --set full summary, NOT a measurement of this run (a run
    under ncu is never a bench run)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as fh:
            j = json.load(fh)
    except Exception:
        return None, None
    v = j.get(workload_name)
    if v is None:
        return None, None
    return v, "committed ncu capture, not this run: profiles/ncu_traffic.json (" + j.get("_source", "") + ")"


def mix_peak(read_fraction):
    """HBM bandwidth at the kernel's read:write mix, from the committed probe
    (profiles/r02_hbm_mix_probe.json: torch kernels of 1R:1W, 2R:1W, 3R:1W,
    read-only and write-only mixes over 4 GiB operands on a B200), linearly
    interpolated between the two nearest measured mixes.  Context beside the
    contract's peak (the 1:1 copy of MEASURED_PEAKS.json), not a replacement:
    a read-heavy kernel can run above the copy figure."""
    p = os.path.join(ROOT, "profiles", "r02_hbm_mix_probe.json")
    try:
        with open(p) as fh:
            cases = json.load(fh)["cases"]
    except Exception:
        return None
    pts = sorted((c["read_fraction"], c["GBps"]) for k, c in cases.items()
                 if 0.0 < c["read_fraction"] < 1.0)  # the mixed cases (the one-sided ones differ in kind)
    if not pts:
        return None
    if read_fraction <= pts[0][0]:
        g = pts[0][1]
    elif read_fraction >= pts[-1][0]:
        g = pts[-1][1]
    else:
        for (f0, g0), (f1, g1) in zip(pts, pts[1:]):
            if f0 <= read_fraction <= f1:
                g = g0 + (g1 - g0) * (read_fraction - f0) / (f1 - f0)
                break
    return {"GBps": g, "read_fraction": read_fraction,
            "source": "profiles/r02_hbm_mix_probe.json (tools/hbm_mix_probe.py; torch kernels, "
                      "interpolated between the nearest mixes; context, not the contract's peak)"}


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.result = None
        if self.proc is None:
            return
        time.sleep(0.15)
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except Exception:
            self.proc.kill()
            out = ""
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if sm:
            self.result = {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx),
                           "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ CPU oracle
def oracle_sample(w, budget_s: float, steps_hint: int | None = None):
    """Time the oracle (as it stands) on a bounded sample of workload w:
    the first rows of the same swarm (same d, objective, parameters), stepping
    `k` iterations.  Returns (rate, seconds, description, (rows, k, sec/step))."""
    import oracle as orc
    rows = 64
    probe = orc.OracleSwarm(rows, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed,
                            vmax=w.vmax)
    t0 = time.perf_counter()
    probe.step(1)
    per_elem = (time.perf_counter() - t0) / (rows * w.d)
    if steps_hint is None:
        k = 5
        rows = max(1, min(w.n, int(budget_s / (per_elem * w.d * k))))
    else:
        k = steps_hint
        rows = max(1, min(w.n, int(budget_s / (per_elem * w.d * k))))
    s = orc.OracleSwarm(rows, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax)
    return s, rows, k


class _PinnedCore:
    """Pin this process to one host core while the oracle is timed (the
    oracle runs single-threaded on one core of the GPU box's host); restored after."""

    def __enter__(self):
        self.core, self.saved = None, None
        try:
            self.saved = os.sched_getaffinity(0)
            self.core = max(self.saved)
            os.sched_setaffinity(0, {self.core})
        except (AttributeError, OSError):
            self.core = None
        return self

    def __exit__(self, *exc):
        if self.saved:
            try:
                os.sched_setaffinity(0, self.saved)
            except OSError:
                pass


def cpu_baseline(w, budget_s: float):
    with _PinnedCore() as pin:
        s, rows, k = oracle_sample(w, budget_s)
        t0 = time.perf_counter()
        s.step(k)
        dt = time.perf_counter() - t0
    rate = rows * w.d * k / dt
    return {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"oracle (single-threaded C++ -O3 -ffp-contract=off) on the first {rows} of "
                      f"{w.n} particles x {w.d} dims, {k} iterations ({dt:.1f} s), create excluded",
            "host_cpu": _cpu_model(), "pinned_core": pin.core}


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip() + f" ({os.cpu_count()} logical cpus)"
    except Exception:
        pass
    return None


def run_reference(args, w):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    K, W = args.steps, args.warmup
    budget = args.ref_seconds  # whole --steps K --warmup W run
    with _PinnedCore() as pin:
        s, rows, _ = oracle_sample(w, budget / max(K + W, 1), steps_hint=1)
        s.step(W)
        t0 = time.perf_counter()
        s.step(K)
        dt = time.perf_counter() - t0
    rate = rows * w.d * K / dt
    sample = (f"oracle (single-threaded C++ -O3 -ffp-contract=off) on the first {rows} of {w.n} "
              f"particles x {w.d} dims; {W} warm-up + {K} timed iterations ({dt:.1f} s)")
    line = {
        "impl": "reference", "metric": METRIC, "value": rate, "unit": UNIT,
        "n_gpus": args.gpus, "steps": K, "warmup": W, "ms_per_step": dt * 1e3 / K,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": _config(w, args.gpus, K, extra={"sample_rows": rows}),
        "cpu_baseline": {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": sample, "host_cpu": _cpu_model(), "pinned_core": pin.core},
        "e2e": {"value": rate, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def _config(w, n_gpus, K, extra=None):
    state = 3 * w.n * w.d * 4
    cfg = {"workload": w.name, "objective": OBJ_NAMES[w.objective], "n": w.n, "d": w.d,
           "w": w.w, "c1": w.c1, "c2": w.c2, "lo": w.lo, "hi": w.hi,
           "vmax": w.vmax if w.vmax > 0 else 1.0, "seed": w.seed, "timed_iterations": K,
           "parallelism": f"particle-split x{n_gpus}" if n_gpus > 1 else "single GPU",
           "l2": ("inputs larger than L2 (%.2f GB state vs 126 MB L2); no flush" % (state / 1e9))
           if state / max(n_gpus, 1) > L2_BYTES else
           ("state (%.1f MB/GPU) fits in L2: L2-resident, not an HBM number" % (state / n_gpus / 1e6))}
    if extra:
        cfg.update(extra)
    return cfg


# ------------------------------------------------------------------ GPU arm
def run_gpu(args, w):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_liuwc21_b200 as fp
    from paper_conf_icpp_liuwc21_b200.distributed import destroy_comm, init_comm

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # PSO_SHARE_GPU=1 (harness test only, never a bench number): every rank runs
    # on GPU 0 -- gloo process group, no NCCL communicator (NCCL refuses two
    # ranks on one device), the NVLink-peer protocol over CUDA IPC between the
    # rank processes.  Exercises the N > 1 code path of this script on one GPU.
    share = world > 1 and os.environ.get("PSO_SHARE_GPU", "0") not in ("", "0")
    if share:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm = None
    # PSO_FORCE_EXCHANGE=1 runs the multi-GPU exchange (process group, NCCL
    # communicator, all-gather + select every step) even on one rank.
    use_comm = world > 1 or os.environ.get("PSO_FORCE_EXCHANGE", "0") not in ("", "0")
    if share:
        dist.init_process_group("gloo")
    elif use_comm:
        if world > 1:  # the communicator setup of every rank stays visible on stderr
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        dist.init_process_group("nccl", device_id=dev)
        comm = init_comm(local)

    def barrier():
        if use_comm:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if share else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def make_swarm(**kw):
        if share:  # communicator-free ranks: world/rank given, init after P2P connect
            s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed,
                         vmax=w.vmax, device=local, stream=stream, world=world, rank=rank,
                         defer_init=True, async_gbest=async_gbest, **kw)
            from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
            if not connect_p2p(s):
                raise SystemExit("PSO_SHARE_GPU: peer mapping failed")
            s.init()
            return s, True
        s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax,
                     device=local, stream=stream, nccl_comm=comm, async_gbest=async_gbest,
                     allreduce_exchange=xmode == "allreduce", **kw)
        # gbest exchange between ranks: NVLink peer stores from the step kernels
        # (default), or the NCCL all-gather (PSO_EXCHANGE=nccl, or if any rank
        # cannot map its peers)
        on = False
        if use_comm and xmode == "p2p":
            from paper_conf_icpp_liuwc21_b200.distributed import connect_p2p
            on = connect_p2p(s)
        return s, on

    # gbest exchange for N > 1: "p2p" NVLink peer stores from the step kernels
    # (default; falls back to the all-gather if any rank cannot map / probe its
    # peers), "nccl" the all-gather, "allreduce" north_star's allreduce-min of the
    # key + bit-exact sum-broadcast of the winner's row
    xmode = os.environ.get("PSO_EXCHANGE", "p2p")
    stream = torch.cuda.Stream(device=dev)  # the library enqueues on this stream
    torch.cuda.set_stream(stream)
    K, W = args.steps, args.warmup
    # PSO_GBEST=async: NEXT-4 asynchronous particle split (peers' records one
    # iteration late); default synchronous (bitwise independent of N)
    async_gbest = use_comm and os.environ.get("PSO_GBEST", "sync") == "async"
    sw, p2p = make_swarm(timing=True)
    # NCCL exchange (fallback): the timed run replays the library's captured
    # [step, all-gather] graphs, which carry no timing events; the step kernel's
    # own duration is then measured on a second handle with per-launch events.
    graphs = use_comm and not p2p and not share
    if graphs:
        sw.close()
        sw, _ = make_swarm(timing=False)
    sw.step(W)
    sw.synchronize()
    sw.reset_counters()

    # ---------------- device-timed region
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        ev0.record(stream)
        sw.step(K)
        ev1.record(stream)
        barrier()
    ms = max_over_ranks(ev0.elapsed_time(ev1))
    info = sw.info()
    if graphs:
        tk, _ = make_swarm(timing=True)
        tk.step(min(K, 100))
        ti = tk.info()
        info["step_kernel_ms"], info["step_kernel_count"] = ti["step_kernel_ms"], ti["step_kernel_count"]
        tk.close()
    kern_ms = max_over_ranks(info["step_kernel_ms"] / max(info["step_kernel_count"], 1))
    launches = int(info["launches"])
    improvements = info["improvements"]
    n_local = info["n_local"]
    gf, gi, _ = sw.gbest(pos=False)

    total_updates = w.n * w.d * K
    value = total_updates / (ms / 1e3)
    rho = improvements / max(n_local * K, 1)
    # algorithmic bytes per launch of the step kernel: x, v read and
    # written every row; pbest rows read / written only where the kernel must
    # (pb_loads / pb_stores counted in-kernel: with lazy pbest rows a row whose
    # pbest equals x skips both); pf read + written on improvement
    pbl = info["pb_loads"] / max(n_local * K, 1)
    pbs = info["pb_stores"] / max(n_local * K, 1)
    if info["resident"] in (1, 2):  # state held in shared memory: no per-iteration row traffic counted
        pbl, pbs = 1.0, rho
    bytes_per_update = 16.0 + 4.0 * pbl + 4.0 * pbs
    alg_bytes = n_local * w.d * bytes_per_update + n_local * (4.0 + 4.0 * rho)
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    # (20 + 4 rho + 8/d) B per update, pbest read for every row
    survey_gbs = n_local * w.d * (20.0 + 4.0 * rho + 8.0 / w.d) / (kern_ms / 1e3) / 1e9
    traffic, traffic_src = ncu_traffic(w.name)
    peak, peak_src = hbm_peak()
    rd = 8.0 + 4.0 * pbl  # bytes read / written per update (x, v; pbest where moved)
    mix = mix_peak(rd / bytes_per_update)
    if mix:
        mix["frac"] = achieved / mix["GBps"]

    # ---------------- end to end through the public API, host buffers
    e2e = None
    clk_e2e = None
    if not args.no_e2e:
        X = torch.empty((n_local, w.d), dtype=torch.float32).pin_memory()
        V = torch.empty_like(X).pin_memory()
        PB = torch.empty_like(X).pin_memory()
        pf = torch.empty((n_local,), dtype=torch.float32).pin_memory()
        _, _, _, _, t_ck = sw.get_state(out=(X, V, PB, pf))  # a host checkpoint of the swarm
        sw.close()
        gpos = torch.empty((w.d,), dtype=torch.float32).pin_memory()

        def e2e_run(per_step: bool):
            s2, _ = make_swarm()
            with ClockSampler(local) as ck:
                barrier()
                t0 = time.perf_counter()
                s2.set_state(X, V, PB, pf, t=t_ck)  # H2D of the whole swarm state
                if per_step:  # every step: pso_step(1) + D2H of its result (gbest fitness, index)
                    for _ in range(K):
                        s2.step(1)
                        s2.gbest(pos=False)
                else:
                    s2.step(K)
                r = s2.gbest(out=gpos)  # D2H of the final gbest position (synchronises)
                barrier()
                sec = max_over_ranks(time.perf_counter() - t0)
            s2.close()
            return sec, r, ck.result

        e2e_s, res, clk_e2e = e2e_run(per_step=True)
        batched_s, _, _ = e2e_run(per_step=False)
        h2d = 3 * n_local * w.d * 4 + n_local * 4
        d2h = K * (4 + 8) + 4 * w.d
        e2e = {"value": total_updates / e2e_s, "unit": UNIT,
               "h2d_bytes_per_step": h2d / K, "d2h_bytes_per_step": d2h / K,
               "seconds": e2e_s,
               "path": ("pso_set_state(pinned host X,V,PB,pf) once, then per step pso_step(1) + "
                        "pso_get_gbest (fitness, index to host), then pso_get_gbest(position)"),
               "batched": {"value": total_updates / batched_s, "seconds": batched_s,
                           "path": "pso_set_state + pso_step(K) + pso_get_gbest(position)"},
               "gbest": res[0]}
    else:
        sw.close()
    if comm:
        destroy_comm(comm)

    line = None
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cpu = cpu_baseline(w, args.cpu_seconds)
        state_per_gpu = 3 * n_local * w.d * 4
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
            "warmup": W, "ms_per_step": ms / K, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (swarm initialised from Philox streams, seed %d)" % w.seed,
            "config": _config(w, world, K, extra={"gbest_exchange": (
                "nvlink-peer-stores" if p2p else
                "nccl-allreduce-min + sum-broadcast (CUDA graph)" if xmode == "allreduce" else
                "nccl-allgather (CUDA graph)") if use_comm else None,
                "gbest_mode": ("async" if async_gbest else "sync") if use_comm else None,
                **({"shared_gpu_harness_test": True} if share else {})}),
            "gpu_launches": launches,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "peak_source": peak_src,
                         "frac_of_spec": achieved / SPEC_HBM_GBS,  # vs the 8 TB/s data-sheet figure
                         "mix_peak": mix,
                         "traffic": traffic, "traffic_source": traffic_src,
                         # SURVEY 8(d)'s accounting: every pbest row read, 4 rho written
                         "frac_survey_formula": survey_gbs / peak,
                         "achieved_survey_formula": survey_gbs,
                         "kernel": ("k_col_step + k_col_decide per iteration (fused move+eval "
                                    "with tile partials, then the pbest/gbest decisions; PDL "
                                    "launches, timed together)" if info["column_split"]
                                    else "k_step (fused move+eval+pbest+gbest)"),
                         "kernel_avg_us": kern_ms * 1e3,
                         "bytes_per_update": bytes_per_update, "rho": rho,
                         "pb_load_frac": pbl, "pb_store_frac": pbs,
                         "lazy_pbest": bool(info["lazy_pb"]),
                         "alg_bytes_per_launch": alg_bytes,
                         "l2_resident": state_per_gpu <= L2_BYTES,
                         "cta": {"threads": info["threads_per_cta"], "vpt": info["vec_per_thread"],
                                 "grid": info["grid"], "ctas_per_sm": info["ctas_per_sm"],
                                 "tma_pipeline": info["tma_pipeline"],
                                 "stages": info["pipeline_stages"],
                                 "smem_bytes": info["smem_bytes"],
                                 "path": _path_name(info)}},
            "clocks": clk.result, "e2e": e2e, "clocks_e2e": clk_e2e,
            "cpu_baseline": cpu, "gbest": {"fitness": gf, "index": gi},
        }
        print(json.dumps(line), flush=True)
    if use_comm:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _free_port() -> int:
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def self_launch(args) -> int:
    """`python bench.py --gpus N` (N > 1) outside torchrun: re-run this script
    as N ranks (one process per GPU) through torch.distributed.run on
    127.0.0.1; rank 0 prints the one JSON line.  NCCL's init lines stay on
    stderr (NCCL_DEBUG=INFO, INIT subsystem) so every rank's communicator
    setup is visible."""
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
           f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    print("[bench] launching %d ranks: %s" % (args.gpus, " ".join(cmd)), file=sys.stderr, flush=True)
    return subprocess.run(cmd, env=env).returncode


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)
    w = WORKLOADS[args.workload]
    if args.impl == "reference":
        return run_reference(args, w)
    return run_gpu(args, w)


if __name__ == "__main__":
    sys.exit(main())
