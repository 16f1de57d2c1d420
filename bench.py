#!/usr/bin/env python
"""Benchmark of the NetAlignBP + matching hot path (BASELINE.json:metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

A "step" is one pass of the per-iteration hot path of Alg. 2:
BP update a3-a6 (iterate) + rounding a7-a8 (two matchings, evaluate, best) on
config O (BASELINE.json:configs[2], ontology-shaped, ~5e6 L edges, ~1e8 nnz(S)),
with S (a2) and the L layouts (a1) built once before timing (they are
"executed only once").  `value` = steps per second =
BP iterations/s; squares/s and the end-to-end align time (init + 100
iterations + best, host buffers, through the C ABI) are reported beside it.

Prints ONE JSON line on rank 0.  See DESIGN.md "Measurement".
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np

METRIC = "BP iterations/sec and squares/sec; end-to-end align time at 1/2/4/8 B200"
UNIT = "iterations/s"
# algorithmic bytes: (2*sigma + 4) per nonzero of S, (9*sigma + 8) per L edge
SIGMA = 8
BYTES_PER_NZ = 2 * SIGMA + 4
BYTES_PER_EDGE = 9 * SIGMA + 8


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def read_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as fh:
            pk = json.load(fh)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """Samples SM clock and throttle reasons via NVML while the timed region runs."""

    def __init__(self, device_index=0, period_s=0.005):
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
            self._ok = True
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
        self.period = period_s
        self._t = None

    def _names(self, mask):
        nv = self._nv
        table = {
            "gpu_idle": getattr(nv, "nvmlClocksEventReasonGpuIdle", 0x1),
            "applications_clocks_setting": getattr(nv, "nvmlClocksEventReasonApplicationsClocksSetting", 0x2),
            "sw_power_cap": getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4),
            "hw_slowdown": getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8),
            "sync_boost": getattr(nv, "nvmlClocksEventReasonSyncBoost", 0x10),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
            "hw_power_brake_slowdown": getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
        }
        return [k for k, v in table.items() if mask & v]

    def _run(self):
        nv = self._nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                try:
                    mask = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                except AttributeError:
                    mask = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self._h)
                for r in self._names(mask):
                    if r != "gpu_idle":
                        self.reasons.add(r)
            except Exception:
                pass
            time.sleep(self.period)

    def start(self):
        if self._ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()

    def stop(self):
        if self._t:
            self._stop.set()
            self._t.join()
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and os.environ.get("CUALIGN_ONE_GPU") == "1":
        # test mode: every rank on cuda:0 (the sandbox has one GPU); a distinct
        # NCCL host id per rank stops NCCL rejecting the shared device, so the
        # ranks connect over its socket transport (timings are not B200 numbers)
        local = 0
        os.environ["NCCL_HOSTID"] = f"cualign-one-gpu-{rank}"
        os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
        os.environ.setdefault("NCCL_IB_DISABLE", "1")
        os.environ.setdefault("NCCL_NVLS_ENABLE", "0")
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        backend = "gloo" if args.impl == "reference" else "nccl"
        if backend == "nccl":
            import torch
            torch.cuda.set_device(local)
        dist.init_process_group(backend=backend)
    return rank, world, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(x, world, device=None):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def host_info():
    """The host the oracle runs on: cores, CPU model, memory."""
    model = None
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    try:
        mem_gb = os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES") / 2 ** 30
    except (ValueError, OSError, AttributeError):
        mem_gb = None
    return {"nproc": os.cpu_count(), "cpu_model": model or platform.processor() or platform.machine(),
            "mem_gib": round(mem_gb, 1) if mem_gb else None}


def oracle_on_O(n_warm, n_steps, pin_core=0):
    """The oracle (oracle/, single-threaded fp64 C, as it stands) on the FULL
    config O instance, pinned to one core: create (S by its definition), then
    n_warm untimed and n_steps timed steps, a step = Alg. 2 l.9-16 + l.17-24
    (step_gamma + round).  Returns a dict of timings."""
    try:
        os.sched_setaffinity(0, {pin_core})
    except (AttributeError, OSError):
        pass
    os.environ["OMP_NUM_THREADS"] = "1"
    from oracle import Oracle
    from synth import make_config
    t0 = time.perf_counter()
    inst = make_config("O")
    t1 = time.perf_counter()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    t2 = time.perf_counter()
    for _ in range(n_warm):
        o.step_gamma(inst.gamma)
        o.round()
    step_s = []
    for _ in range(n_steps):
        ts = time.perf_counter()
        o.step_gamma(inst.gamma)
        o.round()
        step_s.append(time.perf_counter() - ts)
    try:
        cores = len(os.sched_getaffinity(0))
    except (AttributeError, OSError):
        cores = None
    return {"gen_s": t1 - t0, "create_s": t2 - t1, "step_s": step_s, "m": o.m, "s": o.s, "cores": cores,
            "pinned_core": pin_core, "n_warm": n_warm, "n_steps": n_steps, "inst": inst}


def start_oracle_child(n_steps):
    """cpu_baseline leg: the oracle on full O in a child process pinned to core
    0 (OMP_NUM_THREADS=1), running while the GPU is measured (the bench process
    moves to the other cores); collected at the end."""
    env = dict(os.environ, OMP_NUM_THREADS="1")
    env.pop("RANK", None)
    env.pop("WORLD_SIZE", None)
    return subprocess.Popen([sys.executable, os.path.abspath(__file__), "--oracle-child", str(n_steps)],
                            stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True, env=env, cwd=ROOT)


def finish_oracle_child(proc):
    out, err = proc.communicate()
    if proc.returncode != 0:
        return {"value": None, "unit": UNIT, "cores": 1, "kind": "oracle",
                "sample": "failed: " + (err or "")[-300:]}
    d = json.loads(out.strip().splitlines()[-1])
    per = statistics.mean(d["step_s"])
    return {"value": 1.0 / per, "unit": UNIT, "cores": d["cores"], "kind": "oracle",
            "sample": (f"full config O (m={d['m']}, s={d['s']}): oracle create {d['create_s']:.1f} s (untimed), "
                       f"then {d['n_steps']} timed steps of Alg. 2 step + round, single thread pinned to core "
                       f"{d['pinned_core']} (taskset-equivalent sched_setaffinity, OMP_NUM_THREADS=1); "
                       f"value = 1 / mean step time ({per:.3f} s)"),
            "step_s": d["step_s"], "create_s": d["create_s"], "host": host_info()}


def workload_config(name, scale, inst, m, s, world, weak, exact=False, fp32=False):
    """The bench line's `config` (both arms print the same one for the same
    workload)."""
    squares = s // 2
    return {"workload": f"{name}: " + inst.meta["desc"], "scale": scale,
            "n_a": inst.A.n, "n_b": inst.B.n, "m": m, "s": s, "squares": squares,
            "alpha": inst.alpha, "beta": inst.beta, "gamma": inst.gamma,
            "parallelism": (f"A-vertex-block shards x{world} (NCCL)" if world > 1 else "single"),
            "value_unit_note": ("O-equivalent iterations/s: iterations/s x squares / squares(O)"
                                if weak else "iterations/s of this instance"),
            "l2": "inputs larger than L2 (square layout %.2f GB vs 126 MB L2)" % (24 * squares / 1e9),
            "mode": ("exact" if exact else "fast") + ("+fp32S" if fp32 else "")}


def run_reference(args, rank, world):
    """--impl reference: the oracle as it stands on one host core, on the SAME
    workload as our arm (full config O), W warm-up and K timed steps, a step =
    one Alg. 2 iteration + its rounding (no reference implementation exists:
    the reference is a paper).  Rank 0 only; other ranks exit without work."""
    if rank != 0:
        return
    d = oracle_on_O(args.warmup, args.steps)
    total = sum(d["step_s"])
    value = args.steps / total
    sample = (f"full config O (m={d['m']}, s={d['s']}); oracle create {d['create_s']:.1f} s untimed, "
              f"{args.warmup} warm-up + {args.steps} timed steps (Alg. 2 step + round each), single thread "
              f"pinned to core {d['pinned_core']}")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000.0 * total / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": workload_config("O", 1.0, d["inst"], d["m"], d["s"], 1, False),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": d["cores"], "kind": "oracle", "sample": sample,
                             "host": host_info()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def read_peaks_bf16():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            return float(json.load(fh)["bf16_tflops"]), "measured (MEASURED_PEAKS.json bf16_tflops)"
    except Exception:
        return 2250.0, "fallback (nominal dense bf16)"


def knn_measure(ca, dev, peak, n=65536, d=128, k=20, reps=3):
    """NEXT-2: L from embeddings by cualign_knn -- cosine
    similarity tiles on the tcgen05 tensor cores (bf16 in, fp32 accumulate)
    with the fused running top-k.  Device-resident N(0,1) embeddings; the
    whole call (prep, similarity + top-k, merge) timed with CUDA events;
    dense-equivalent 2 n^2 d flop per call against the measured bf16 peak."""
    import torch
    g = torch.Generator(device=f"cuda:{dev}").manual_seed(20231112)
    YA = torch.randn(n, d, device=f"cuda:{dev}", generator=g)
    YB = torch.randn(n, d, device=f"cuda:{dev}", generator=g)
    ca.knn(YA, YB, k, device=dev)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        ca.knn(YA, YB, k, device=dev)
    e1.record()
    torch.cuda.synchronize()
    sec = e0.elapsed_time(e1) / 1e3 / reps
    tf = 2.0 * n * n * d / sec / 1e12
    return {"workload": f"n_A = n_B = {n}, d = {d}, top-{k}, N(0,1) embeddings", "s_per_call": sec,
            "roofline": {"bound": "tensor", "achieved": tf, "peak": peak[0], "unit": "TFLOP/s",
                         "frac": tf / peak[0], "peak_source": peak[1]}}


def launch_floor_ms(n_kernels, reps=200):
    """Graph-replay floor of a step of n_kernels tiny kernels: a CUDA graph of
    n_kernels one-element torch kernels, replayed, CUDA-event timed."""
    import torch
    x = torch.zeros(1, device="cuda")
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        for _ in range(3):
            x.add_(1.0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(n_kernels):
                x.add_(1.0)
        for _ in range(10):
            g.replay()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(reps):
            g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def config_point(ca, name, k, steps, stream, dev):
    """One BASELINE.json config on one GPU: generate (seeded),
    init through the C ABI, warm-up steps, then
    `steps` device-timed steps (iteration + rounding) on the launching stream;
    iterate-only and round-only graph replays with per-kernel event nodes for
    the split and the square pass's HBM fraction (20 B per nonzero of S)."""
    import torch
    from synth import make_config
    t0 = time.perf_counter()
    inst = make_config(name, k=k)
    row = {"n_a": inst.A.n, "n_b": inst.B.n, "m": int(inst.L.m), "gen_s": round(time.perf_counter() - t0, 1),
           "desc": inst.meta["desc"] + (f" (k = {k})" if k else "")}
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, device=dev, stream=stream)
    torch.cuda.synchronize()
    row["init_s"] = time.perf_counter() - t0
    peak, _ = read_peaks()
    with h:
        sz = h.sizes()
        s_nz = int(sz["s"])
        row.update(s=s_nz, squares=s_nz // 2, device_gb=round(sz["device_bytes"] / 1e9, 2))
        h.run(10)
        torch.cuda.synchronize()
        h.stats(reset=True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h.run(steps)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / steps
        st = h.stats(reset=True)
        kernels = st["launches"] / steps
        row.update(steps=steps, ms_per_step=ms, iters_per_s=1e3 / ms, squares_per_s=(s_nz / 2) * 1e3 / ms,
                   kernels_per_step=kernels,
                   schedule={1: "pipelined", 2: "serial", 0: "forked"}.get(h.sizes()["schedule"], "?"))
        h.set_timing(True)
        h.run(steps, with_round=False)
        torch.cuda.synchronize()
        it = {c: v / steps for c, v in h.stats(reset=True)["class_ms"].items() if v}
        h.run(steps, with_round=True, iterate=False)
        torch.cuda.synchronize()
        rd = {c: v / steps for c, v in h.stats(reset=True)["class_ms"].items() if v}
        h.set_timing(False)
        bp_ms = sum(it.values())
        alg = BYTES_PER_NZ * s_nz + BYTES_PER_EDGE * row["m"]
        row.update(bp_ms=bp_ms, round_ms=sum(rd.values()), iterate_kernel_ms=it, round_kernel_ms=rd,
                   iteration_hbm_frac=alg / (bp_ms * 1e-3) / 1e9 / peak)
        if it.get("square"):
            row["square_hbm_frac"] = BYTES_PER_NZ * s_nz / (it["square"] * 1e-3) / 1e9 / peak
    if name in ("T", "P"):
        # latency-bound working sets: against the graph-replay floor
        fl = launch_floor_ms(int(round(kernels)))
        row["graph_replay_floor_ms"] = fl
        row["floor_frac"] = fl / ms
    return row


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default=None,
                    help="workload: O at N = 1 (BASELINE.json configs[2]); S sharded at N > 1 (configs[3])")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--e2e-iters", type=int, default=100)
    ap.add_argument("--e2e-reps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--oracle-steps", type=int, default=3, help="timed oracle steps of the cpu_baseline leg")
    ap.add_argument("--oracle-child", type=int, default=None, help=argparse.SUPPRESS)
    ap.add_argument("--no-configs", action="store_true", help="skip the T/P/S/R sub-measurements")
    ap.add_argument("--config-points", default="T,P,S,R5,R50")
    ap.add_argument("--config-steps", type=int, default=20)
    ap.add_argument("--exact", action="store_true", help="CUALIGN_FLAG_EXACT (oracle-order sums)")
    ap.add_argument("--fp32", action="store_true", help="CUALIGN_FLAG_FP32_S (S^p stored in fp32, NEXT-3)")
    ap.add_argument("--match-rounds", action="store_true", help="pointer-round matching schedule")
    ap.add_argument("--schedule", type=int, default=0,
                    help="step schedule (cualign_params.schedule: 0 the library's rule, 1 pipelined, 2 serial, 3 forked)")
    ap.add_argument("--prof-steps", type=int, default=20, help="steps of the per-kernel timing pass")
    ap.add_argument("--strong", action="store_true", help="N > 1: shard the same instance (strong scaling)")
    ap.add_argument("--no-knn", action="store_true", help="skip the NEXT-2 kNN measurement")
    args = ap.parse_args()
    if args.oracle_child is not None:
        d = oracle_on_O(0, args.oracle_child)
        d.pop("inst")
        print(json.dumps(d), flush=True)
        return
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    rank, world, local = dist_setup(args)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if args.config is None:
        args.config = "O" if world == 1 else "S"
    if world > 1 and args.config == "S":
        args.strong = True  # configs[3]: one instance sharded over the N GPUs
    # cpu_baseline: the oracle on full O in a child pinned to core 0, running
    # while the GPU is measured; this process keeps off that core
    oracle_proc = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and args.config == "O" and args.scale == 1.0:
        oracle_proc = start_oracle_child(args.oracle_steps)
        try:
            others = set(range(os.cpu_count() or 1)) - {0}
            if others:
                os.sched_setaffinity(0, others)
        except (AttributeError, OSError):
            pass

    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config

    dev = local
    torch.cuda.set_device(dev)
    # N > 1: config S (BASELINE.json configs[3], "sharded across 2/4/8 B200")
    # split by A-vertex blocks over the N ranks, strong scaling;
    # --config O at N > 1: weak scaling, the O generator at N x the size.
    # Every rank generates the identical seeded instance.
    scale = args.scale * (world if (world > 1 and not args.strong) else 1)
    t_gen = time.perf_counter()
    inst = make_config(args.config, scale=scale, seed=None)
    t_gen = time.perf_counter() - t_gen
    log(f"[rank {rank}] generated {args.config} (scale {scale}) in {t_gen:.1f}s: "
        f"n_A={inst.A.n} n_B={inst.B.n} m={inst.L.m}")

    def shard_kw():
        if world == 1:
            return {}
        import torch.distributed as dist
        obj = [ca.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        return dict(world=world, rank=rank, nccl_id=obj[0])
    # a dedicated stream: the library launches on it and the timing events are
    # recorded on it (torch's default stream is the legacy stream, which does
    # not order against the library's non-blocking streams)
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    flags = (ca.FLAG_EXACT if args.exact else 0) | (ca.FLAG_MATCH_ROUNDS if args.match_rounds else 0) | \
        (ca.FLAG_FP32_S if args.fp32 else 0)
    bytes_per_nz = (2 * 4 + 4) if args.fp32 else BYTES_PER_NZ  # S^p pair stored as 2 x fp32

    # ---------------------------------------------------------------- init
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags=flags, schedule=args.schedule,
                     device=dev, stream=stream, **shard_kw())
    torch.cuda.synchronize()
    init_s = max_over_ranks(time.perf_counter() - t0, world, device=f"cuda:{dev}")
    sz = h.sizes()
    m, s, squares = sz["m"], sz["s"], sz["squares"]
    s_local = 2 * sz["squares_local"]  # this rank's share of the square pass
    log(f"[rank {rank}] init {init_s:.3f}s s={s} squares={squares} max_row={sz['max_row']} "
        f"fp_bits={sz['fixed_point_bits']} device_bytes={sz['device_bytes']/1e9:.2f}GB")

    # ------------------------------------------------------------- warmup
    # (each step = iterate(1) + round, replayed from the library's CUDA graph;
    # the library's step schedule comes from its size rule, no timed selection)
    h.run(args.warmup)
    torch.cuda.synchronize()
    h.stats(reset=True)
    barrier(world)

    # --------------------------------------------------------- timed region
    sampler = ClockSampler(dev)
    sampler.start()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    barrier(world)
    ev0.record(stream)
    h.run(args.steps)
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier(world)
    clocks = sampler.stop()
    elapsed_ms = ev0.elapsed_time(ev1)
    elapsed_ms = max_over_ranks(elapsed_ms, world, device=f"cuda:{dev}")
    st = h.stats(reset=True)
    _, info = h.get_best()
    step_schedule = {-1: "undecided", 0: "rounding forked beside the square pass", 1: "pipelined",
                     2: "serial"}.get(h.sizes()["schedule"], "?")

    # ----------------------------------------------- per-kernel timing pass
    # event-record nodes inside the captured step graph, read after each replay
    prof_steps = max(1, min(args.prof_steps, args.steps))
    h.set_timing(True)
    h.run(prof_steps)
    h.set_timing(False)
    torch.cuda.synchronize()
    pst = h.stats(reset=True)

    # isolated per-kernel timing (no concurrent rounding branch): iterate-only
    # and round-only graph replays after the timed region, each kernel's
    # algorithmic bytes against the measured HBM peak
    iso = None
    if world == 1:
        h.set_timing(True)
        h.run(prof_steps, with_round=False)
        torch.cuda.synchronize()
        ist = h.stats(reset=True)
        h.run(prof_steps, with_round=True, iterate=False)
        torch.cuda.synchronize()
        rst = h.stats(reset=True)
        h.set_timing(False)
        nA_, nB_ = inst.A.n, inst.B.n
        kbytes = {"square": bytes_per_nz * s_local,
                  # La, Lb, w, y^p, z^p, F-sum read; y^p, z^p, y^c, z^c, d, u, F-sum written
                  "edge": (8 + 4 * 8 + 7 * 8) * m,
                  # y^p by A rows, B incidence ids + z^p gathers, row pointers, (max1, max2) out
                  "top2": (8 + 4 + 8) * m + 8 * (nA_ + nB_) + 16 * (nA_ + nB_)}
        peak_i, _ = read_peaks()
        iso = {}
        for name in ("top2", "edge", "square"):
            ms_k = ist["class_ms"][name] / max(ist["class_launches"][name], 1)
            iso[name] = {"ms": ms_k, "alg_bytes": kbytes[name],
                         "frac_hbm": (kbytes[name] / (ms_k * 1e-3) / 1e9 / peak_i) if ms_k > 0 else None}
        for name in ("match", "eval", "matchaux", "other"):
            iso[name] = {"ms": rst["class_ms"][name] / prof_steps}
        it_ms = sum(iso[k]["ms"] for k in ("top2", "edge", "square")) + ist["class_ms"]["other"] / prof_steps
        it_alg = bytes_per_nz * s_local + BYTES_PER_EDGE * m
        iso["iteration"] = {"ms": it_ms, "alg_bytes": it_alg, "frac_hbm": it_alg / (it_ms * 1e-3) / 1e9 / peak_i}
        iso["round_ms"] = sum(iso[k]["ms"] for k in ("match", "eval", "matchaux", "other"))

    # sharded: the exchanges of one step: bytes each rank
    # receives (counted by the library per collective) against NVLink 5's
    # 900 GB/s per direction, time from events around the exchanges
    exchange = None
    if world > 1:
        x_bytes = max_over_ranks(st["comm_bytes_in"] / args.steps, world, device=f"cuda:{dev}")
        x_ms = max_over_ranks(pst["comm_ms"] / prof_steps, world, device=f"cuda:{dev}")
        x_gbs = x_bytes / (x_ms * 1e-3) / 1e9 if x_ms > 0 else None
        exchange = {"bytes_in_per_iter_per_rank": x_bytes, "calls_per_iter": st["comm_calls"] / args.steps,
                    "ms_per_iter": x_ms, "achieved": x_gbs, "peak": 900.0, "unit": "GB/s",
                    "frac": (x_gbs / 900.0) if x_gbs else None,
                    "transport": ("NCCL socket transport, all ranks on one GPU (CUALIGN_ONE_GPU=1): "
                                  "not an NVLink number" if os.environ.get("CUALIGN_ONE_GPU") == "1"
                                  else "NCCL (NVLink / NVSwitch)")}

    # value: iterations/s of the instance; weak scaling (O x N) in
    # O-equivalent iterations/s (iterations/s x squares / squares of one O),
    # i.e. the whole job's throughput in units of the N = 1 workload
    from synth import O_full_work
    weak = world > 1 and not args.strong
    unit_squares = O_full_work()[1] / 2 if (args.config == "O" and args.scale == 1.0) else squares / max(world, 1)
    work_units = squares / unit_squares if weak else 1.0
    value = args.steps * work_units / (elapsed_ms / 1e3)
    ms_per_step = elapsed_ms / args.steps
    cls_ms = pst["class_ms"]
    cls_n = pst["class_launches"]
    sq_ms = cls_ms["square"] / prof_steps  # per step (a sharded step runs it in two ranges)
    bp_ms = (cls_ms["top2"] + cls_ms["edge"] + cls_ms["square"] + cls_ms["rowsum"] + cls_ms["other"]) / prof_steps
    round_ms = (cls_ms["match"] + cls_ms["eval"] + cls_ms["matchaux"]) / prof_steps
    peak, peak_src = read_peaks()
    sq_bytes = bytes_per_nz * s_local              # algorithmic bytes of one (this rank's) square-pass launch
    sq_gbs = sq_bytes / (sq_ms * 1e-3) / 1e9 if sq_ms > 0 else 0.0
    it_bytes = bytes_per_nz * s_local + BYTES_PER_EDGE * (sz["edge_end"] - sz["edge_begin"])
    it_gbs = it_bytes / (bp_ms * 1e-3) / 1e9 if bp_ms > 0 else 0.0
    # DRAM traffic needs a profiler pass (ncu dram__bytes), which this timed
    # run cannot take: null here; the ncu --set full captures are in profiles/
    traffic = None

    # ------------------------------------------------------------------ e2e
    e2e = None
    align_time_s = None
    if not args.no_e2e:
        # pinned host buffers, the public API (C ABI), H2D of all inputs and
        # D2H of every round's info and of the best matching inside the region
        def pin(x):
            return torch.from_numpy(np.ascontiguousarray(x)).pin_memory()

        class G:  # graph with pinned arrays
            pass

        GA, GB, GL = G(), G(), G()
        GA.n, GA.rowptr, GA.col = inst.A.n, pin(inst.A.rowptr), pin(inst.A.col)
        GB.n, GB.rowptr, GB.col = inst.B.n, pin(inst.B.rowptr), pin(inst.B.col)
        GL.a, GL.b, GL.w = pin(inst.L.a), pin(inst.L.b), pin(inst.L.w)
        h2d = sum(int(t.numel() * t.element_size()) for t in
                  (GA.rowptr, GA.col, GB.rowptr, GB.col, GL.a, GL.b, GL.w))
        del h
        torch.cuda.empty_cache()
        # E2E_REPS complete alignments (each: new handle, inputs from the host,
        # result to the host), the median reported (wall clock is exposed to
        # host-side hiccups; every run's time is listed)
        runs = []
        for _ in range(max(1, args.e2e_reps)):
            torch.cuda.synchronize()
            barrier(world)
            t0 = time.perf_counter()
            mate, binfo, infos = ca.align(GA, GB, GL, inst.alpha, inst.beta, inst.gamma, n_iter=args.e2e_iters,
                                          flags=flags, device=dev, stream=stream, **shard_kw())
            torch.cuda.synchronize()
            t_done = time.perf_counter()
            # end-to-end = inputs on the host -> best matching on the host; the
            # handle's teardown after the result is reported separately
            runs.append((max_over_ranks(binfo["t_result"] - t0, world, device=f"cuda:{dev}"),
                         t_done - binfo["t_result"], binfo))
        runs.sort(key=lambda r: r[0])
        align_time_s, teardown_s, binfo = runs[len(runs) // 2]
        # device time of the same e2e_iters steps from p = 0 on a fresh handle
        # (CUDA events, no host copies): the iterations phase's floor -- early
        # iterations differ from the steady state the timed region measures
        dev_iter_s = None
        if world == 1:
            with ca.CuAlignBP(GA, GB, GL, inst.alpha, inst.beta, inst.gamma, flags=flags, device=dev,
                              stream=stream) as hf:
                torch.cuda.synchronize()
                f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                f0.record(stream)
                hf.run(args.e2e_iters)
                f1.record(stream)
                torch.cuda.synchronize()
                dev_iter_s = f0.elapsed_time(f1) / 1e3
        d2h = args.e2e_iters * 112 + 4 * inst.A.n
        e2e = {"value": args.e2e_iters * work_units / align_time_s, "unit": UNIT,
               "h2d_bytes_per_step": h2d / args.e2e_iters, "d2h_bytes_per_step": d2h / args.e2e_iters,
               "align_time_s": align_time_s, "teardown_s": teardown_s, "iters": args.e2e_iters,
               "phases_s": binfo.get("phases_s"), "schedule": binfo.get("schedule"),
               "align_times_s": [r[0] for r in runs], "timing": f"median of {len(runs)} alignments",
               "best_score": binfo["best_score"], "best_iter": binfo["best_iter"],
               "iterations_device_s": dev_iter_s}
        if rank == 0:
            # NEXT-4: quality of the best alignment against the generator's ground truth
            try:
                qd = ca.quality(inst.A, inst.B, ca.alignment_map(mate, inst.L),
                                np.asarray(inst.truth, dtype=np.int32), device=dev)
                e2e["quality"] = {k: qd[k] for k in ("nc", "ec", "ics", "s3", "ncv", "ncv_gs3")}
            except Exception as ex:  # pragma: no cover
                e2e["quality"] = {"error": str(ex)}
    else:
        del h

    # --------------------------------------------------------- cpu baseline
    # ------------------------------------------------ other configs (T/P/S/R)
    configs = None
    if rank == 0 and world == 1 and not args.no_configs:
        configs = {}
        for pt in [x for x in args.config_points.split(",") if x]:
            name, k = pt[0], (int(pt[1:]) if len(pt) > 1 else None)
            try:
                configs[pt] = config_point(ca, name, k, args.config_steps, stream, dev)
            except Exception as ex:  # pragma: no cover
                configs[pt] = {"error": str(ex)[:300]}
            log(f"[config {pt}] {json.dumps(configs[pt])[:300]}")
            torch.cuda.empty_cache()

    cpu = finish_oracle_child(oracle_proc) if oracle_proc is not None else None

    # ------------------------------------------- NEXT-2: kNN on the tensor cores
    knn = None
    if rank == 0 and world == 1 and not args.no_knn:
        try:
            knn = knn_measure(ca, dev, read_peaks_bf16())
        except Exception as e:  # pragma: no cover
            knn = {"error": str(e)}

    if rank != 0:
        return
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong" if (world > 1 and args.strong) else "weak", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": workload_config(args.config, args.scale, inst, m, s, world, weak, args.exact, args.fp32),
        "squares_per_s": squares * args.steps / (elapsed_ms / 1e3),
        "bp_iters_per_s": 1e3 / bp_ms if bp_ms > 0 else None,
        "round_ms": round_ms, "bp_ms": bp_ms, "init_s": init_s,
        "roofline": {"bound": "hbm", "kernel": "k_square (a3+a5+a6 square pass)",
                     "achieved": sq_gbs, "peak": peak, "unit": "GB/s", "frac": sq_gbs / peak,
                     "traffic": traffic, "alg_bytes_per_launch": sq_bytes,
                     "launch_ms": sq_ms, "peak_source": peak_src},
        "iteration_roofline": {"achieved": it_gbs, "frac": it_gbs / peak, "alg_bytes": it_bytes,
                               "bp_ms": bp_ms},
        "kernel_ms_per_step": {k: v / prof_steps for k, v in cls_ms.items() if v},
        "kernels_isolated": iso,
        "exchange": exchange,
        "kernel_timing": (f"CUDA event-record nodes around each kernel inside the captured step "
                          f"graph, {prof_steps} steps after the timed region"),
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": st["launches"],
        "clocks": clocks,
        "best_score": info["best_score"],
        "last_round": {k: info[k] for k in ("iter", "card_y", "card_z", "overlap_y", "overlap_z",
                                            "rounds_y", "rounds_z", "score")},
        "match_schedule": "rounds" if args.match_rounds else "suitor",
        "step_schedule": step_schedule,
        "next2_knn": knn,
        "configs": configs,
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
    try:
        import torch.distributed as dist
        if dist.is_available() and dist.is_initialized():
            dist.destroy_process_group()
    except Exception:  # pragma: no cover
        pass
