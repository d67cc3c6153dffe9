#!/usr/bin/env python
"""bench.py -- the driver's benchmark contract for this repo.

Workload (BASELINE.json configs[1]): 4th-order 3D stencil, 256^3 fp64, specialized on
dims and coeffs through libproteus, z-slab halo exchange at N > 1 GPUs (fused into the
kernel over peer memory, or NCCL).  One "step" = one sweep of the whole hot path:
proteus_launch (key -> hash -> in-memory hit -> cuLaunchKernelEx) of the specialized
stencil4_ws cubin over the full field (+ halo exchange when N > 1).  The JIT compile happens once, in the untimed warm-up; the cold/warm
end-to-end jobs that INCLUDE the JIT time are measured separately and reported under
"speedup_vs_aot" (the first half of the BASELINE metric).

value  = algorithmic HBM bytes of all ranks per second (16 B per grid point per sweep:
         read u once, write w once) over K timed sweeps, CUDA events, max over ranks.
e2e    = the same metric for a job as a user runs it through the public API: the input
         slab is copied from pinned host memory, K sweeps run through proteus_launch with
         the state resident on the device (the field is the solver's state, as weights are
         a trainer's), every sweep's result probe (one fp64 of the new field) is read back
         to the host, and the result slab is copied back -- all inside the timed region;
         h2d/d2h_bytes_per_step = those bytes / K.  "e2e_full_roundtrip" additionally
         reports the extreme case of copying the whole slab in and out around EVERY sweep.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--job-sweeps T] [--n 256]
Under torchrun (N > 1) every rank runs its slab; rank 0 prints the JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import shutil
import statistics
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# NVRTC results would otherwise be cached by the driver's ComputeCache (~/.nv) across
# processes and runs, hiding the real compile cost from "cold" measurements.
os.environ.setdefault("CUDA_CACHE_DISABLE", "1")

METRIC = "speedup vs AOT sm_100a incl. JIT time; specialized-kernel HBM GB/s vs peak"


def workload_name(n):
    """config.workload, identical in both arms (the kernel is named separately)."""
    return f"CFG 2: 13-point 4th-order 3D stencil {n}^3 fp64, one sweep per step"
BYTES_PER_POINT = 16


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", "--field-n", dest="n", type=int, default=256,
                    help="global field is n^3 (--field-n: the same, for torchrun command lines, "
                         "where --n is an ambiguous abbreviation of torchrun's own options)")
    ap.add_argument("--job-sweeps", type=int, default=10000,
                    help="sweeps of the end-to-end AOT-vs-JIT jobs (SURVEY.md §8d-2 headline)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-e2e-jobs", action="store_true")
    ap.add_argument("--e2e-processes", type=int, default=5,
                    help="N=1: runs per variant of the fresh-process end-to-end jobs (0 = skip)")
    ap.add_argument("--e2e-probe", default="side", choices=["side", "inline"],
                    help="e2e: per-sweep probe D2H on a copy stream (side) or inline")
    ap.add_argument("--workload", default="stencil", choices=["stencil", "adam"],
                    help="stencil: CFG 2 (the driver's line); adam: CFG 1 sharded over ranks "
                         "(SURVEY §8e, no collective), one adam_run launch of --adam-steps "
                         "steps per bench step")
    ap.add_argument("--adam-n", type=int, default=10 ** 6)
    ap.add_argument("--adam-steps", type=int, default=100)
    ap.add_argument("--kernel", default="stencil4_ws", choices=["stencil4_ws", "stencil4"],
                    help="stencil4_ws: warp-specialized TMA ring (default); stencil4: v3")
    ap.add_argument("--no-suite", dest="suite", action="store_false",
                    help="skip the CFG 1/3/4/5 'suite' key of the N=1 line")
    ap.add_argument("--dump-final", default=None,
                    help="after the run, each rank writes its owned planes after "
                         "--dump-sweeps fresh sweeps to <path>.rank<r>.npy (tests)")
    ap.add_argument("--dump-sweeps", type=int, default=7)
    ap.add_argument("--halo", default="p2p", choices=["p2p", "nccl"],
                    help="N > 1: p2p = halo stores fused into stencil4_p2p over CUDA-IPC peer "
                         "memory + stream flags (default); nccl = batch_isend_irecv")
    return ap.parse_args()


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def ncu_traffic(kernel):
    """dram read+write bytes per launch from the committed ncu --set full summary."""
    path = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(path) as f:
            return json.load(f).get(kernel)
    except Exception:
        return None


class ClockSampler:
    """SM clocks and throttle reasons sampled (NVML, every 20 ms) during the timed
    region, as B200_PROFILING.md's clocks line asks."""

    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
               0x4: "sw_power_cap"}

    def __init__(self, cuda_index):
        self.idx = cuda_index
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        if vis:
            try:
                self.idx = int(vis.split(",")[cuda_index])
            except ValueError:
                pass
        self.samples = []
        self.stop = threading.Event()
        self.ready = threading.Event()
        self.smax = None
        self.err = None

    def _run(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.idx)
            self.smax = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            get_reasons = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                nv.nvmlDeviceGetCurrentClocksThrottleReasons
            while True:
                self.samples.append((nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM), get_reasons(h)))
                self.ready.set()
                if self.stop.wait(0.02):
                    break
            self.samples.append((nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM), get_reasons(h)))
        except Exception as e:  # pragma: no cover
            self.err = repr(e)
        finally:
            self.ready.set()

    def __enter__(self):
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        self.ready.wait(timeout=10)   # first sample taken before the timed region starts
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=5)

    def summary(self):
        sm = [s for s, _ in self.samples]
        reasons = set()
        for _, mask in self.samples:
            for bit, name in self.REASONS.items():
                if mask & bit:
                    reasons.add(name)
        d = {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.smax,
             "reasons": sorted(reasons), "samples": len(sm)}
        if self.err:
            d["error"] = self.err
        return d


def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


# ------------------------------------------------------------------------- reference arm
def run_reference(args, world, rank):
    """The oracle (plain C, OpenMP over z-planes) timed on this host's cores on the same
    workload; bounded sample: as many full 256^3 sweeps as fit in ~cpu_seconds."""
    if rank != 0:
        return
    import numpy as np

    import oracle
    import synthetic
    oracle.build()
    cores = len(os.sched_getaffinity(0))
    oracle.set_threads(cores)
    n = args.n
    u0 = synthetic.stencil_inputs(n, n, n)
    co = synthetic.STENCIL_COEFFS
    a = np.ascontiguousarray(u0)
    b = np.empty_like(a)
    lib = oracle.lib()
    p = lambda x: x.ctypes.data_as(__import__("ctypes").c_void_p)
    for _ in range(max(1, args.warmup // 5)):
        lib.oracle_stencil_sweep(p(a), p(b), n, n, n, *co)
    sweeps, t0 = 0, time.perf_counter()
    steps = max(1, args.steps)
    times = []
    while sweeps < steps:
        ts = time.perf_counter()
        lib.oracle_stencil_sweep(p(a), p(b), n, n, n, *co)
        a, b = b, a
        times.append(time.perf_counter() - ts)
        sweeps += 1
        if time.perf_counter() - t0 > args.cpu_seconds and sweeps >= 2:
            break
    el = time.perf_counter() - t0
    gbs = sweeps * n ** 3 * BYTES_PER_POINT / el / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(gbs, 3), "unit": "GB/s",
            "n_gpus": world, "steps": sweeps, "warmup": args.warmup,
            "ms_per_step": round(el / sweeps * 1e3, 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(n), "global_points": n ** 3,
                       "kernel": "oracle_stencil_sweep (plain C, OpenMP over z-planes)",
                       "sweeps_timed": sweeps},
            "cpu_baseline": {"value": round(gbs, 3), "unit": "GB/s", "cores": cores,
                             "kind": "oracle",
                             "sample": f"{sweeps} full {n}^3 sweeps (~{args.cpu_seconds:.0f} s bound)"},
            "e2e": {"value": round(gbs, 3), "unit": "GB/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------- our arm
def main():
    args = parse()
    world, rank, local = dist_setup(args)
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    import numpy as np
    import torch

    import synthetic
    from paper_conf_cgo_georgakoudispb25_b200 import halo
    from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W

    # BENCH_SHARE_GPU=1 (testing the N > 1 path on a 1-GPU box): ranks share the visible
    # devices round-robin and the process group uses gloo instead of NCCL.
    share = os.environ.get("BENCH_SHARE_GPU") == "1"
    if share:
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    torch.zeros(1, device=dev)
    group = None
    if world > 1:
        import torch.distributed as dist
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
        # who runs where (stderr; stdout carries only the JSON line): the driver can check
        # that N ranks came up, each on its own GPU, and which backend moves the halos
        props = torch.cuda.get_device_properties(dev)
        where = [None] * world
        dist.all_gather_object(where, (rank, local, str(getattr(props, "uuid", props.name))))
        if rank == 0:
            nccl_v = None if share else ".".join(map(str, torch.cuda.nccl.version()))
            print(f"[bench] world={world} backend={dist.get_backend()} nccl={nccl_v} "
                  f"distinct_gpus={len(set(w[2] for w in where))} ranks={where}",
                  file=sys.stderr, flush=True)

    def barrier():
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return float(t.item())

    if args.workload == "adam":
        return run_adam(args, world, rank, local, dev, barrier, max_over_ranks)

    n = args.n
    assert n % world == 0
    nzl = n // world
    co = synthetic.STENCIL_COEFFS
    u0 = synthetic.stencil_inputs(n, n, n)
    lo, hi = rank * nzl - 2, (rank + 1) * nzl + 2
    slab_np = np.zeros((nzl + 4, n, n))
    s0, s1 = max(lo, 0), min(hi, n)
    slab_np[s0 - lo:s1 - lo] = u0[s0:s1]
    del u0
    slab_host = torch.from_numpy(slab_np).pin_memory()
    cache_root = tempfile.mkdtemp(prefix=f"proteus-bench-r{rank}-")

    def fresh_slab():
        return slab_host.to(dev, non_blocking=False)

    use_p2p = world > 1 and args.halo == "p2p"
    halo_note = "p2p" if use_p2p else (("gloo (host-staged; ranks share a GPU)" if share
                                        else "nccl") if world > 1 else "none")

    def all_ranks_ok(ok):
        t = torch.tensor([1 if ok else 0], dtype=torch.int32, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MIN)
        return bool(t.item())

    if use_p2p:
        # one arena (both slabs + flags) per rank, mapped by the neighbours once (CUDA IPC)
        why = ""
        ref_backend = "gloo (host-staged)" if share else "NCCL"
        try:
            parts = halo.p2p_arena(n, n, nzl, dev)
            P.proteus_init(device=local, cache_dir=os.path.join(cache_root, "ipc"), mode="all")
            p2p_left, p2p_right, _opened = halo.connect_ipc(parts[0], rank, world, group)
            # validate the fused path against the process-group exchange on this machine
            # (NCCL; gloo with host staging when ranks share a GPU): 3 sweeps each, generic
            # kernels (same arithmetic), bit-identical slabs on every rank
            st = halo.P2PZSlabStencil(W.register("stencil4_p2p"), parts, nx=n, ny=n, nzl=nzl,
                                      nzg=n, rank=rank, world=world, coeffs=co, left=p2p_left,
                                      right=p2p_right, variant="aot")
            parts[1].copy_(slab_host)
            parts[2].copy_(parts[1])
            parts[3].zero_()
            barrier()
            for _ in range(3):
                st.sweep()
            ref = halo.ZSlabStencil(W.register("stencil4_ws"), slab_host.to(dev), nx=n, ny=n,
                                    nzl=nzl, nzg=n, rank=rank, world=world, coeffs=co,
                                    group=group, variant="aot")
            for _ in range(3):
                ref.sweep()
            torch.cuda.synchronize()
            own = slice(2, nzl + 2)
            ok = torch.equal(st.current[own], ref.current[own])
            why = "" if ok else f"fused halo differs from the {ref_backend} exchange"
            del st, ref
        except Exception as e:   # pragma: no cover - depends on the machine
            ok, why = False, f"{type(e).__name__}: {e}"[:200]
        P.proteus_finalize()
        if not all_ranks_ok(ok):
            use_p2p = False
            halo_note = f"nccl (fused p2p halo unavailable on this machine: {why or 'another rank'})"
            if rank == 0:
                print(f"[bench] {halo_note}", file=sys.stderr)
        else:
            halo_note = f"p2p (validated bit-exact against the {ref_backend} exchange, 3 sweeps)"
    kname = "stencil4_p2p" if use_p2p else args.kernel

    def make_stencil(k, variant):
        """This rank's distributed stencil over fresh copies of the input slab."""
        if use_p2p:
            parts[1].copy_(slab_host)
            parts[2].copy_(parts[1])
            parts[3].zero_()
            barrier()                 # every rank reset its flags before anyone signals
            return halo.P2PZSlabStencil(k, parts, nx=n, ny=n, nzl=nzl, nzg=n, rank=rank,
                                        world=world, coeffs=co, left=p2p_left, right=p2p_right,
                                        variant=variant)
        return halo.ZSlabStencil(k, fresh_slab(), nx=n, ny=n, nzl=nzl, nzg=n, rank=rank,
                                 world=world, coeffs=co, group=group, variant=variant)

    # ---------------- end-to-end jobs incl. JIT (cold / warm cache) vs AOT ----------
    speed = {}
    job_T = args.job_sweeps
    if not args.no_e2e_jobs:
        def job(variant, cache_dir, async_workers=0):
            """init -> register -> T sweeps -> sync; host wall time."""
            if use_p2p:
                parts[1].copy_(slab_host)
                parts[2].copy_(parts[1])
                parts[3].zero_()
            else:
                slab = fresh_slab()
            barrier()
            t0 = time.perf_counter()
            P.proteus_init(device=local, cache_dir=cache_dir, mode="all",
                           async_workers=async_workers)
            k = W.register(kname)
            if use_p2p:
                st = halo.P2PZSlabStencil(k, parts, nx=n, ny=n, nzl=nzl, nzg=n, rank=rank,
                                          world=world, coeffs=co, left=p2p_left,
                                          right=p2p_right, variant=variant)
            else:
                st = halo.ZSlabStencil(k, slab, nx=n, ny=n, nzl=nzl, nzg=n, rank=rank,
                                       world=world, coeffs=co, group=group, variant=variant)
            for _ in range(job_T):
                st.sweep()
            torch.cuda.synchronize()
            el = time.perf_counter() - t0
            stats = P.proteus_cache_stats()
            P.proteus_finalize()
            return max_over_ranks(el), stats

        # Order matters: the cold job is the process's FIRST proteus_init, so it pays the
        # NVRTC initialisation a fresh process pays (with CUDA_CACHE_DISABLE=1 nothing is
        # served from the driver's cache); the empty persistent dir makes it a true miss.
        jdir = os.path.join(cache_root, "job")
        t_cold, st_cold = job("jit", jdir)              # cold process-level JIT
        t_aot, _ = job("aot", jdir)                     # generic AOT sm_100a
        t_aot = min(t_aot, job("aot", jdir)[0])
        t_warm, st_warm = job("jit", jdir)              # populated cache ("Proteus+$")
        shutil.rmtree(jdir, ignore_errors=True)
        t_async, st_async = job("jit", jdir, async_workers=2)   # empty dir, generic meanwhile
        shutil.rmtree(jdir, ignore_errors=True)
        t_cold2, st_cold2 = job("jit", jdir)            # empty dir, compiler already up
        speed = {"job_sweeps": job_T, "aot_s": round(t_aot, 4), "jit_cold_s": round(t_cold, 4),
                 "jit_warm_s": round(t_warm, 4),
                 "cold_incl_jit": round(t_aot / t_cold, 4),
                 "warm_disk_cache": round(t_aot / t_warm, 4),
                 "jit_cold_warm_compiler_s": round(t_cold2, 4),
                 "cold_warm_compiler": round(t_aot / t_cold2, 4),
                 "jit_async_cold_s": round(t_async, 4),
                 "cold_async_incl_jit": round(t_aot / t_async, 4),
                 "async_generic_launches": st_async["generic_launches"],
                 "jit_compile_ms_warm_compiler": round(st_cold2["compile_ms_total"], 2),
                 "jit_compile_ms": round(st_cold["compile_ms_total"], 2),
                 "disk_load_ms": round(st_warm["load_ms_total"], 3),
                 "cold_compiles": st_cold["compiles"], "warm_disk_hits": st_warm["disk_hits"]}

    # ---------------- steady state: K timed sweeps through the hot cache ------------
    P.proteus_init(device=local, cache_dir=os.path.join(cache_root, "steady"), mode="all")
    k = W.register(kname)
    st = make_stencil(k, "jit")
    stream = torch.cuda.current_stream()
    for _ in range(max(3, args.warmup)):
        st.sweep()
    barrier()

    # ---------------- kernel-only speedup (AOT generic vs JIT, same launches) -------
    def timed_sweeps(variant, reps=50):
        st.variant = variant
        for _ in range(5):
            st.sweep()
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(reps):
            st.sweep()
        b.record(stream)
        barrier()
        st.variant = "jit"
        return max_over_ranks(a.elapsed_time(b) / reps)

    # measured before the long timed loop, alternating the variants (3 rounds x 200 sweeps,
    # median per variant): right after the 3000-sweep loop the GPU runs power-capped for a
    # while and the AOT kernel (two waves, the more latency-sensitive) read 10-20% slow,
    # biasing kernel_only upwards (1.36 vs 1.22 in the suite's cool measurement)
    rounds = {"aot": [], "jit": []}
    for _ in range(3):
        for variant in ("aot", "jit"):
            rounds[variant].append(timed_sweeps(variant, reps=200))
    t_k_aot = statistics.median(rounds["aot"])
    t_k_jit = statistics.median(rounds["jit"])
    speed["kernel_only"] = round(t_k_aot / t_k_jit, 4)
    speed["aot_sweep_us"] = round(t_k_aot * 1e3, 2)
    speed["jit_sweep_us"] = round(t_k_jit * 1e3, 2)
    if speed.get("jit_compile_ms") is not None and t_k_aot > t_k_jit:
        speed["break_even_sweeps"] = round(speed["jit_compile_ms"] / (t_k_aot - t_k_jit), 1)

    launches_per_step = 1 if (world == 1 or use_p2p) else 3
    # N = 1: one launch per step, so the kernel's average launch duration is the timed
    # region / steps (no per-step events, which would add gaps).  N > 1: events bracket
    # the compute launches of each step (boundary + interior, before the halo wait).
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)] if world > 1 else None
    with ClockSampler(local) as clk:
        # the W warm-up sweeps again right before the timed region: the sampler's NVML
        # start-up idles the GPU for ~0.1 s, and a short timed region (K = 20 is 0.9 ms)
        # would otherwise start on a clock still ramping back up (r02bi: 47.3 us per sweep
        # at K = 20 against 46.1 at K = 3000, SM clock median 1848 vs 1965 MHz)
        for _ in range(max(3, args.warmup)):
            st.sweep()
        stats0 = P.proteus_cache_stats()
        barrier()
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_start.record(stream)
        for i in range(args.steps):
            st.sweep(events=ev[i] if ev else None)
        t_end.record(stream)
        barrier()
    stats1 = P.proteus_cache_stats()
    ms = t_start.elapsed_time(t_end)
    ms = max_over_ranks(ms)
    step_ms = ms / args.steps
    total_bytes = n ** 3 * BYTES_PER_POINT          # all ranks, one sweep
    value = total_bytes * args.steps / (ms / 1e3) / 1e9
    if world == 1:
        kern_ms = step_ms
    else:
        kern_ms = max_over_ranks(statistics.mean(a.elapsed_time(b) for a, b in ev))
    kern_bytes = nzl * n * n * BYTES_PER_POINT      # this rank's launches per step
    peak, peak_kind = measured_peaks()
    achieved = kern_bytes / (kern_ms / 1e3) / 1e9
    assert stats1["mem_hits"] - stats0["mem_hits"] == args.steps * launches_per_step, (stats0, stats1)
    assert stats1["compiles"] == stats0["compiles"]

    # ---------------- cache-hit launch latency (host), tiny kernel ------------------
    kd = W.register("daxpy")
    x = torch.ones(256, dtype=torch.float64, device=dev)
    y = torch.zeros_like(x)
    Ld = W.daxpy_launch(kd, 1.0, x, y)
    Ld.jit()
    torch.cuda.synchronize()
    lat = {}
    for variant in ("aot", "jit"):
        f = Ld.aot if variant == "aot" else Ld.jit
        best = []
        for _ in range(5):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(200):
                f()
            best.append((time.perf_counter() - t0) / 200 * 1e6)
            torch.cuda.synchronize()
        lat[variant] = min(best)
    speed["hit_launch_us"] = round(lat["jit"], 3)
    speed["aot_launch_us"] = round(lat["aot"], 3)
    speed["hit_overhead_us"] = round(lat["jit"] - lat["aot"], 3)

    # ---------------- e2e through host buffers --------------------------------------
    out_host = torch.empty_like(slab_host).pin_memory()
    slab_bytes = slab_host.numel() * 8
    st.variant = "jit"
    # (a) the job: slab in, K sweeps with a per-sweep probe read back, slab out
    e2e_steps = args.steps
    probe_host = torch.empty(e2e_steps, dtype=torch.float64).pin_memory()
    probe_at = (2 + nzl // 2) * n * n + (n // 2) * n + n // 2     # mid-slab interior point
    # Probe read-back: "side" copies each sweep's probe on a copy stream that waits for that
    # sweep (event), so the 8-B D2H does not sit between two sweeps of the compute stream
    # (it would serialize them and cancel the programmatic-dependent-launch overlap); the
    # sweep that overwrites a probed buffer (two sweeps later, ping-pong) waits for the
    # copy.  "inline" copies on the compute stream.
    main = torch.cuda.current_stream()
    side = torch.cuda.Stream()
    swept = [torch.cuda.Event() for _ in range(2)]
    copied = [torch.cuda.Event() for _ in range(2)]
    barrier()
    t0 = time.perf_counter()
    st.current.copy_(slab_host, non_blocking=True)
    for i in range(e2e_steps):
        if args.e2e_probe == "side" and i >= 2:
            main.wait_event(copied[i % 2])      # the buffer this sweep writes was probed
        st.sweep()
        probe_src = st.current.view(-1)[probe_at:probe_at + 1]
        if args.e2e_probe == "side":
            swept[i % 2].record(main)
            side.wait_event(swept[i % 2])
            with torch.cuda.stream(side):
                probe_host[i:i + 1].copy_(probe_src, non_blocking=True)
            copied[i % 2].record(side)
        else:
            probe_host[i:i + 1].copy_(probe_src, non_blocking=True)
    main.wait_stream(side)
    out_host.copy_(st.current, non_blocking=True)
    torch.cuda.synchronize()
    e2e_s = max_over_ranks(time.perf_counter() - t0)
    # the last probe read back is the probed point of the result slab
    assert probe_host[e2e_steps - 1].item() == out_host.view(-1)[probe_at].item()
    e2e_value = total_bytes * e2e_steps / e2e_s / 1e9
    e2e_h2d = slab_bytes / e2e_steps
    e2e_d2h = (slab_bytes + 8 * e2e_steps) / e2e_steps
    # (b) extreme case: the whole slab in and out around every sweep
    rt_steps = max(3, min(args.steps, 20))
    barrier()
    t0 = time.perf_counter()
    for _ in range(rt_steps):
        st.current.copy_(slab_host, non_blocking=True)
        st.sweep()
        out_host.copy_(st.current, non_blocking=True)
    torch.cuda.synchronize()
    rt_s = max_over_ranks(time.perf_counter() - t0)
    rt_value = total_bytes * rt_steps / rt_s / 1e9

    launches_timed = args.steps * launches_per_step
    if args.dump_final:
        # fresh input, --dump-sweeps sweeps through the same path, owned planes to disk
        # (tests/test_gpu_bench_multirank.py compares them with the oracle)
        import numpy as np
        fin = make_stencil(k, "jit")
        for _ in range(args.dump_sweeps):
            fin.sweep()
        torch.cuda.synchronize()
        np.save(f"{args.dump_final}.rank{rank}.npy", fin.current[2:nzl + 2].cpu().numpy())
        barrier()
    P.proteus_finalize()
    shutil.rmtree(cache_root, ignore_errors=True)

    if rank == 0:
        cpu = cpu_baseline(args, world)
        suite = None
        if world == 1 and args.suite:
            # CFG 1, 3, 4, 5 beside the CFG 2 line (bench_suite.driver_suite): AOT vs JIT
            # step times, roofline fractions, NVRTC ms, oracle spot checks in the CPU leg
            try:
                import bench_suite
                tmps = tempfile.mkdtemp(prefix="proteus-bench-suite-")
                suite = bench_suite.driver_suite(tmps)
                shutil.rmtree(tmps, ignore_errors=True)
            except Exception as e:   # reported, never fatal to the bench line
                suite = {"error": repr(e)[:300]}
        if world == 1 and not args.no_e2e_jobs and args.e2e_processes > 0:
            # the paper's protocol for the headline speedup: every run a fresh process (cold:
            # empty cache dir, NVRTC initialised inside the timed job; warm: the dir the cold
            # run filled), 1 discarded warm-up process, mean +- RSE (bench_suite.py)
            try:
                import bench_suite
                tmpd = tempfile.mkdtemp(prefix="proteus-bench-proc-")
                pr = bench_suite.e2e_processes("stencil", tmpd, runs=args.e2e_processes)
                shutil.rmtree(tmpd, ignore_errors=True)
                speed["fresh_processes"] = {
                    "runs": pr["processes_per_variant"], "job_sweeps": 10000,
                    "variant_orders": pr["variant_orders"],
                    "aot_s": pr["aot_s"], "cold_s": pr["cold_s"],
                    "warm_s": pr["warm_s"], "async_s": pr["async_s"],
                    "cold_incl_jit": pr["speedup_cold"], "warm_disk_cache": pr["speedup_warm"],
                    "cold_async_incl_jit": pr["speedup_async"],
                    "cold_compile_ms": pr["cold_compile_ms"],
                    "rse_flagged": pr["rse_flagged"],
                    # the same job in THIS process (its first proteus_init: NVRTC initialised
                    # inside the timed job), beside the fresh-process means
                    "in_process_first_init_cold_incl_jit": speed.get("cold_incl_jit")}
            except Exception as e:   # reported, never fatal to the bench line
                speed["fresh_processes"] = {"error": repr(e)[:300]}
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(step_ms, 5),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(n),
                       "kernel": f"{kname}, specialized on nx, ny, nzl, nzg, a0, a1, a2 + "
                                 f"launch bounds + dims",
                       "global_points": n ** 3, "slab_planes_per_rank": nzl,
                       "parallelism": f"z-slab x{world}" + ((" + halo fused into the kernel (P2P stores, "
                                                           "stream flags)" if use_p2p else
                                                           f" + {halo_note} halo") if world > 1 else ""),
                       "l2": "working set 256 MiB > 126 MB L2 (no flush needed)",
                       "halo": halo_note,
                       "launch": W.stencil_config(kname)},
            "roofline": {"bound": "hbm", "achieved": round(achieved, 2), "peak": peak,
                         "unit": "GB/s", "frac": round(achieved / peak, 4),
                         "peak_kind": peak_kind, "kernel": f"{kname} (JIT)",
                         "traffic": ncu_traffic(kname),
                         "algorithmic_bytes_per_launch": kern_bytes,
                         "kernel_ms": round(kern_ms, 5)},
            "speedup_vs_aot": speed,
            "cpu_baseline": cpu,
            "e2e": {"value": round(e2e_value, 3), "unit": "GB/s",
                    "h2d_bytes_per_step": round(e2e_h2d, 1),
                    "d2h_bytes_per_step": round(e2e_d2h, 1), "steps": e2e_steps,
                    "job": "slab H2D, K sweeps via proteus_launch each with an 8-B probe D2H, "
                           "slab D2H", "probe": args.e2e_probe},
            "e2e_full_roundtrip": {"value": round(rt_value, 3), "unit": "GB/s",
                                   "h2d_bytes_per_step": slab_bytes,
                                   "d2h_bytes_per_step": slab_bytes, "steps": rt_steps},
            "gpu_launches": launches_timed,
            "clocks": clk.summary(),
        }
        if suite is not None:
            line["suite"] = suite
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def run_adam(args, world, rank, local, dev, barrier, max_over_ranks):
    """CFG 1 over parameter shards: rank r updates its contiguous,
    16-B aligned slice of the 10^6 parameters with adam_run (the paper's kernel form: the
    time loop inside one launch, R-adam-4); no collective -- barriers bracket the timing
    only.  value = all ranks' param-steps per second (max over ranks of the device time)."""
    import torch

    import synthetic
    from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    from paper_conf_cgo_georgakoudispb25_b200.shard import shard_range

    n, steps = args.adam_n, args.adam_steps
    lo, hi = shard_range(n, world, rank)
    S = synthetic.ADAM_SCALARS
    sc = dict(lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"],
              decay=S["decay"], steps=steps)
    host = [torch.from_numpy(a[lo:hi].copy()).pin_memory() for a in synthetic.adam_inputs(n)]
    t = [h.to(dev) for h in host]
    cache_root = tempfile.mkdtemp(prefix=f"proteus-bench-adam-r{rank}-")
    P.proteus_init(device=local, cache_dir=cache_root, mode="all")
    k = W.register("adam_run")
    L = W.adam_run_launch(k, *t, **sc) if hi > lo else None

    def launch():
        if L is not None:
            L("jit")

    for _ in range(args.warmup):           # includes the JIT compile of this shard's n
        launch()
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        e0.record(stream)
        for _ in range(args.steps):
            launch()
        e1.record(stream)
        barrier()
    ms = max_over_ranks(e0.elapsed_time(e1) / args.steps)
    value = n * steps / (ms / 1e3)
    # e2e: shard H2D from pinned memory, K launches each with the first parameter of the
    # shard read back (side stream, event-ordered), shard D2H
    probe = torch.empty(args.steps, dtype=torch.float32).pin_memory()
    side = torch.cuda.Stream()
    ev = torch.cuda.Event()
    out = [torch.empty_like(h).pin_memory() for h in host[:3]]
    barrier()
    t0 = time.perf_counter()
    for d, h in zip(t, host):
        d.copy_(h, non_blocking=True)
    for i in range(args.steps):
        launch()
        if hi > lo:
            ev.record(stream)
            side.wait_event(ev)
            with torch.cuda.stream(side):
                probe[i:i + 1].copy_(t[0][:1], non_blocking=True)
            stream.wait_stream(side)      # the next launch overwrites p
    for o, d in zip(out, t[:3]):
        o.copy_(d, non_blocking=True)
    torch.cuda.synchronize()
    e2e_s = max_over_ranks(time.perf_counter() - t0)
    nbytes = sum(h.numel() * 4 for h in host)
    st = P.proteus_cache_stats()
    P.proteus_finalize()
    shutil.rmtree(cache_root, ignore_errors=True)
    if rank != 0:
        return
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    sm_mhz = float(peaks.get("sm_max_mhz", 1965.0))
    issue_peak = 148 * 4 * sm_mhz * 1e6          # warp instructions / s
    # per launch of one rank's shard (rank 0 holds the largest shard; ms is the max over ranks)
    inst = (ncu_traffic("adam_run_warp_inst") or 0.0) * ((hi - lo) / 10 ** 6) * (steps / 100)
    # the SFU bounds adam_run since the folded step (DESIGN.md R-adam-6)
    sfu = (hi - lo) * steps * W.ADAM_RUN_SFU_PER_ELEMENT_STEP[synthetic.ADAM_SCALARS["mode"]]
    sfu_pk = W.sfu_peak(sm_mhz)
    line = {
        "metric": "fused Adam param-steps/s (CFG 1, parameter shards, no collective)",
        "value": round(value, 1), "unit": "param-steps/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 5),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": f"CFG 1: fused Adam, {n} fp32 params, {steps} steps per launch",
                   "kernel": "adam_run, specialized on n, lr, b1, b2, eps, grad_scale, decay, "
                             "steps + launch bounds + dims",
                   "parallelism": f"parameter shards x{world}", "shard_rank0": [0, shard_range(n, world, 0)[1]],
                   "l2": "working set 16 MB, L2-resident by design (the run keeps p/m/v in "
                         "registers; 28 B/param per launch)",
                   "note": "each bench step re-runs steps 1..K of the bias-correction table"},
        "roofline": {"bound": "sfu", "achieved": round(sfu / (ms / 1e3) / 1e9, 2),
                     "peak": round(sfu_pk / 1e9, 2), "unit": "G SFU ops/s",
                     "frac": round(sfu / (ms / 1e3) / sfu_pk, 4),
                     "issue_frac": round(inst / (ms / 1e3) / issue_peak, 4) if inst else None,
                     "traffic": None,
                     "source": "SFU ops per launch of rank 0's shard = params x steps x "
                               "W.ADAM_RUN_SFU_PER_ELEMENT_STEP (sqrt + rcp, = ncu's XU-pipe "
                               "utilisation); peak = 148 SMs x 16 XU lanes x max SM clock; "
                               "issue_frac from ncu warp instructions (profiles/traffic.json "
                               "adam_run_warp_inst, scaled) over 148 x 4 schedulers x clock"},
        "e2e": {"value": round(n * steps * args.steps / e2e_s, 1), "unit": "param-steps/s",
                "h2d_bytes_per_step": round(nbytes * world / args.steps, 1),
                "d2h_bytes_per_step": round((nbytes * 3 / 4 * world + 4 * args.steps) / args.steps, 1)},
        "gpu_launches": args.steps if hi > lo else 0,
        "jit": {"compiles": st["compiles"], "compile_ms": round(st["compile_ms_total"], 2)},
        "clocks": clk.summary(),
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(args, world):
    if world != 1:
        return None
    import ctypes

    import numpy as np

    import oracle
    import synthetic
    try:
        oracle.build()
    except Exception as e:  # pragma: no cover
        return {"error": str(e)}
    cores = len(os.sched_getaffinity(0))
    oracle.set_threads(cores)
    n = args.n
    a = np.ascontiguousarray(synthetic.stencil_inputs(n, n, n))
    b = np.empty_like(a)
    p = lambda x: x.ctypes.data_as(ctypes.c_void_p)
    lib = oracle.lib()
    co = synthetic.STENCIL_COEFFS
    lib.oracle_stencil_sweep(p(a), p(b), n, n, n, *co)
    t0 = time.perf_counter()
    sweeps = 0
    while True:
        lib.oracle_stencil_sweep(p(a), p(b), n, n, n, *co)
        a, b = b, a
        sweeps += 1
        if time.perf_counter() - t0 > args.cpu_seconds:
            break
    el = time.perf_counter() - t0
    # also the oracle on one thread (a bounded sample: 2 sweeps)
    oracle.set_threads(1)
    t1 = time.perf_counter()
    for _ in range(2):
        lib.oracle_stencil_sweep(p(a), p(b), n, n, n, *co)
        a, b = b, a
    el1 = time.perf_counter() - t1
    oracle.set_threads(cores)
    return {"value": round(sweeps * n ** 3 * BYTES_PER_POINT / el / 1e9, 3), "unit": "GB/s",
            "cores": cores, "kind": "oracle",
            "sample": f"{sweeps} full {n}^3 sweeps in {el:.1f} s (OpenMP over z-planes)",
            "single_thread": {"value": round(2 * n ** 3 * BYTES_PER_POINT / el1 / 1e9, 3),
                              "sample": f"2 full {n}^3 sweeps in {el1:.1f} s, 1 thread"},
            "cpu_model": cpu_model()}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


if __name__ == "__main__":
    main()
