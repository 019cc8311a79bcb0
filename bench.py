#!/usr/bin/env python
"""bench.py -- the driver's benchmark contract for the Lime map/reduce hot path on B200.

Headline (BASELINE.json metric "map elements/s (N-body interactions/s) and % of FP32/HBM
roofline, 1-8 B200", config 5): N-Body 2^20 bodies fp32; one STEP = one task-graph pass of the
paper's N-Body: all-gather of positions (NCCL, N > 1) -> force map
(lime_map_nbody) -> integrator (lime_map_nbody_integrate). Strong scaling: the 2^20-body
problem is split by target index over N ranks (torchrun, one process per GPU).

    python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--no-extras] [--no-sharded]

Rank 0 prints ONE JSON line. At every N it carries `sharded_configs`: configs 2-4 partitioned over
the N ranks as SURVEY.md §8(e) says (Black-Scholes strong + weak with an all_reduce, Mandelbrot
cyclic rows, matmul row blocks), each timed as the max over ranks. At N = 1 the line also carries
`configs`: every BASELINE.json configuration and the F-rows measured in the same run (N-Body 4096,
Black-Scholes map and fused map+reduce, Mandelbrot, matmul, reductions, ...), each with its own
roofline.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402

METRIC = "N-body interactions/s (map elements/s)"
UNIT = "interactions/s"
EPS2, DT = 1e-4, 1e-3
FLOP_PER_INTERACTION = 20          # GPU Gems 3 convention
FP32_LANE_OPS_PER_INTERACTION = 12  # 3 FADD + 3 FFMA (r^2) + 3 FMUL + 3 FFMA (acc)
# mass-uniform splits (R11; the equal-mass workload): the mass factors out of each chunk
# sum, 2 FMUL instead of 3 -> 11 FP32 lane-ops per interaction (the 20-flop convention is unchanged)
FP32_LANE_OPS_UNIFORM_MASS = 11
SM_MAX_MHZ_NOMINAL = 1965.0
SMS_B200 = 148
IDEA_SASS_PER_UNIT = 663           # idea_kernel loop: SASS instructions per 16-byte unit (2 blocks)


# ----------------------------------------------------------------------------- peaks
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained", d["bf16_tflops"]),
                "sm_max_mhz": d.get("sm_max_mhz", SM_MAX_MHZ_NOMINAL), "source": "measured (MEASURED_PEAKS.json)"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
            "sm_max_mhz": SM_MAX_MHZ_NOMINAL, "source": "fallback (B200_PROFILING.md)"}


def fp32_peak_tflops(sm_mhz: float) -> float:
    """FP32 FMA peak derived from unit counts: 148 SMs x 128 FP32 lanes x
    2 flop x clock. The step-0 microbenchmark measured 124.9-127.9 lane-ops/clk/SM (profiles/)."""
    return SMS_B200 * 128 * 2 * sm_mhz * 1e6 / 1e12


def ncu_traffic(name: str):
    """dram read+write bytes per launch from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        return json.load(f).get(name)


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled every 200 ms during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.gpu)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except (OSError, FileNotFoundError):
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, pw, reasons = [], None, [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
                pw.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s in sm if s > 0.5 * (mx or 1)] or sm
        return {"sm_mhz": float(np.median(loaded)) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm), "power_w_max": max(pw) if pw else None}


# ----------------------------------------------------------------------------- timing helpers
def flush_l2(buf):
    buf.fill_(1)   # write > L2 (2x l2CacheSize) so the next launch starts cold


_CLEAN = {}


def flush_l2_clean(buf):
    """Write > L2 (the contract's flush), then read a second buffer > L2 so the dirty lines the
    write left behind are written back BEFORE the timed launch (tools/hbm_probe.cu measured the
    write-back of a write-only flush at ~4 us inside a 35-us streaming kernel,
    profiles/experiments/hbm_probe_r01.jsonl); the L2 then holds clean lines of an unrelated buffer."""
    buf.fill_(1)
    key = (buf.device, buf.numel())
    if key not in _CLEAN:
        _CLEAN[key] = torch.zeros(buf.numel() // 4, dtype=torch.int32, device=buf.device)
    torch.amax(_CLEAN[key])


# GPU-side idle before each timed launch: while the device sleeps the host enqueues the start
# event and the launch, so host-side Python/ctypes time never lands between the two events
# (~100 us at 1.9 GHz; outside the event pair).
SLEEP_CYCLES = 200_000


def time_launches(fn, iters, warmup, flush_buf=None, writes_output=False):
    """Median/mean device time of `fn` over `iters` launches, each bracketed by CUDA events on the
    current stream; the L2 is flushed before every launch, outside the event pair, followed by a
    short device sleep so the launch is queued before the start event.

    The flush leaves the L2 in the state the same kernel would leave it in when run back to back
    (none of its own data cached): for a kernel whose output exceeds the L2 (`writes_output`) that
    is FULL OF DIRTY LINES (write-only flush) -- otherwise up to an L2 of its own output would still
    sit unwritten in L2 at the end event and the kernel would be timed without that write-back; for
    a read-mostly kernel it is clean (write, then read another 2x L2 buffer)."""
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(iters)]
    for a, b in ev:
        if flush_buf is not None:
            if writes_output:
                flush_l2(flush_buf)
            else:
                flush_l2_clean(flush_buf)
        torch.cuda._sleep(SLEEP_CYCLES)
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    ms = [a.elapsed_time(b) for a, b in ev]
    return float(np.median(ms)), float(np.mean(ms))


def time_back_to_back(fns, reps, batches, flush_buf=None):
    """Steady-state device time per launch: `reps` launches back to back between one CUDA-event
    pair (cycling through `fns`, each over its own input set, so consecutive launches never reuse
    data: the contract's "inputs larger than L2"), median over `batches`; each batch starts after
    an L2 flush and a device sleep. Amortises the ~1-2 us event-timer granularity and launch
    latency that dominate a single ~40-us launch, and every launch pays the write-back its
    predecessor left in L2, as in a production loop."""
    for f in fns:
        f()
    torch.cuda.synchronize()
    res = []
    for _ in range(batches):
        if flush_buf is not None:
            flush_l2_clean(flush_buf)
        torch.cuda._sleep(SLEEP_CYCLES)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for k in range(reps):
            fns[k % len(fns)]()
        b.record()
        torch.cuda.synchronize()
        res.append(a.elapsed_time(b) / reps)
    return float(np.median(res))


# ----------------------------------------------------------------------------- dist
def dist_init(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and not dist.is_initialized():
        if args.impl == "reference":
            return rank, world, local
        # LIME_DIST_BACKEND=gloo lets several ranks share one GPU to exercise the multi-rank code
        # path where only one GPU is available (NCCL needs one GPU per rank); not for timing.
        backend = os.environ.get("LIME_DIST_BACKEND", "nccl")
        local = local % max(torch.cuda.device_count(), 1)
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    elif torch.cuda.is_available():
        torch.cuda.set_device(local)
    return rank, world, local


def barrier(world):
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()


def max_over_ranks(x: float, world: int) -> float:
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ----------------------------------------------------------------------------- headline
def run_nbody(args, rank, world, local):
    n = args.n
    bodies = torch.from_numpy(inputs.nbody_bodies(n, seed=5))
    sim = ldist.NBodySim(bodies, EPS2, DT, f"cuda:{local}")
    props = torch.cuda.get_device_properties(local)
    flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()

    for _ in range(args.warmup):
        sim.step()
    barrier(world)

    clocks = ClockSampler(local).start()
    f_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier(world)
    t0.record(stream)
    for k in range(args.steps):
        flush_l2(flush)
        sim.gather()
        f_ev[k][0].record(stream)
        sim.force_fn(sim.pos_full, sim.begin, sim.count, sim.eps2, sim.accel)
        f_ev[k][1].record(stream)
        sim.integrate_fn(sim.pos, sim.vel, sim.accel, sim.dt)
    t1.record(stream)
    barrier(world)
    clk = clocks.stop()
    ms_local = t0.elapsed_time(t1)
    force_ms = float(np.mean([a.elapsed_time(b) for a, b in f_ev]))
    ms_total = max_over_ranks(ms_local, world)
    force_ms_max = max_over_ranks(force_ms, world)

    interactions_per_step = float(n) * n
    value = interactions_per_step * args.steps / (ms_total * 1e-3)

    # momentum check (all_reduce of sum m v): |P| / sum m |v| (diagnostic, tiny)
    mom = sim.momentum()
    # e2e: host (pinned) state in/out every step through the public API
    e2e = run_nbody_e2e(args, sim, bodies, world, local)

    peak = fp32_peak_tflops(SM_MAX_MHZ_NOMINAL)
    per_launch_interactions = float(sim.count) * n
    achieved = FLOP_PER_INTERACTION * per_launch_interactions / (force_ms * 1e-3) / 1e12
    obs_mhz = clk.get("sm_mhz") or SM_MAX_MHZ_NOMINAL
    uniform_mass = bool(torch.all(bodies[:, 3] == bodies[0, 3]).item())
    lane_ops = FP32_LANE_OPS_UNIFORM_MASS if uniform_mass else FP32_LANE_OPS_PER_INTERACTION
    pipe_frac = (lane_ops * per_launch_interactions / (force_ms * 1e-3)) / (SMS_B200 * 128 * obs_mhz * 1e6)
    roofline = {"kernel": "lime::nbody::force_kernel", "bound": "alu", "achieved": achieved, "peak": peak,
                "unit": "TFLOP/s", "frac": achieved / peak, "traffic": ncu_traffic("nbody_force_1m"),
                "peak_source": "derived: 148 SM x 128 FP32 lanes x 2 flop x 1965 MHz (microbench: 124.9-127.9 lane-ops/clk/SM)",
                "flop_per_interaction": FLOP_PER_INTERACTION,
                "fp32_lane_ops_per_interaction": lane_ops,
                "element_form": ("mass factored out of each chunk sum (equal masses, DESIGN.md R11; the unequal-mass "
                                 "number at this size is configs.nbody_1m_mixed_masses)" if uniform_mass
                                 else "per-body mass multiply"),
                "fp32_pipe_frac_at_observed_clock": pipe_frac, "observed_sm_mhz": obs_mhz,
                "force_ms_per_launch": force_ms, "force_ms_per_launch_max_rank": force_ms_max,
                "force_share_of_step": force_ms / (ms_local / args.steps)}
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_total / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": headline_config(n, world),
            "roofline": roofline, "e2e": e2e, "gpu_launches": (4 if n > 8192 else 2) * args.steps + (args.steps if world > 1 else 0), "clocks": clk,
            "momentum_residual": float(mom.norm().item())}
    return line


def run_nbody_e2e(args, sim, bodies, world, local):
    n = args.n
    count = sim.count
    if world == 1:
        h_pos = bodies.clone().pin_memory()
        h_vel = torch.zeros((n, 4), dtype=torch.float32).pin_memory()
        step = lambda: lime.nbody_simulate_host(h_pos, h_vel, 1, EPS2, DT, device=f"cuda:{local}")
    else:
        h_pos = sim.pos.cpu().pin_memory()
        h_vel = sim.vel.cpu().pin_memory()
        step = lambda: sim.step_host(h_pos, h_vel)
    for _ in range(max(1, args.warmup)):
        step()
    barrier(world)
    stream = torch.cuda.current_stream()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(args.steps):
        step()
    b.record(stream)
    barrier(world)
    ms = max_over_ranks(a.elapsed_time(b), world)
    return {"value": float(n) * n * args.steps / (ms * 1e-3), "unit": UNIT,
            "h2d_bytes_per_step": 2 * count * 16, "d2h_bytes_per_step": 2 * count * 16,
            "api": "lime_nbody_simulate_host (C ABI, pinned host buffers)" if world == 1
            else "dist.NBodySim.step_host (pinned host shards) + C ABI"}


# ----------------------------------------------------------------------------- other configs (N = 1)
def run_extras(peaks, flush):
    out = {}
    hbm = peaks["hbm_gbs"]
    fp32 = fp32_peak_tflops(SM_MAX_MHZ_NOMINAL)

    # config 1: N-Body 4096, one force launch (latency-bound; split-j fills the GPU)
    b = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
    acc = torch.empty_like(b)
    med, mean = time_launches(lambda: lime.map_nbody(b, EPS2, out=acc), 50, 5, flush)
    inter = 4096.0 * 4096
    ach = FLOP_PER_INTERACTION * inter / (med * 1e-3) / 1e12
    out["nbody_4096"] = {"workload": "configs[0]: N-body 4096 bodies fp32, 1 step force map", "value": inter / (med * 1e-3),
                         "unit": "interactions/s", "ms_per_launch": med,
                         "roofline": {"bound": "alu", "achieved": ach, "peak": fp32, "unit": "TFLOP/s", "frac": ach / fp32,
                                      "traffic": ncu_traffic("nbody_force_4096")}}
    del b, acc
    # the same step in a simulation loop: 100 force + integrate steps captured in one CUDA graph
    sim4k = ldist.NBodySim(torch.from_numpy(inputs.nbody_bodies(4096, seed=1)), EPS2, DT, "cuda")
    g4k = sim4k.capture(100)
    med, _ = time_launches(g4k.replay, 10, 2, flush)
    out["nbody_4096_graph"] = {"workload": "configs[0]: N-body 4096, 100 steps (force map with the integrator fused in, "
                                           "lime_map_nbody_step) per CUDA-graph replay",
                               "value": inter * 100 / (med * 1e-3), "unit": "interactions/s",
                               "ms_per_step": med / 100,
                               "roofline": {"bound": "alu", "achieved": FLOP_PER_INTERACTION * inter * 100 / (med * 1e-3) / 1e12,
                                            "peak": fp32, "unit": "TFLOP/s",
                                            "frac": FLOP_PER_INTERACTION * inter * 100 / (med * 1e-3) / 1e12 / fp32,
                                            "traffic": None}}
    del sim4k, g4k
    # ... and as one persistent cooperative launch (lime_nbody_simulate: grid barrier between steps)
    p4k = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
    v4k = torch.zeros_like(p4k)
    med, _ = time_launches(lambda: lime.nbody_simulate(p4k, v4k, 100, EPS2, DT), 10, 2, flush)
    ach = FLOP_PER_INTERACTION * inter * 100 / (med * 1e-3) / 1e12
    out["nbody_4096_simulate"] = {"workload": "configs[0]: N-body 4096, 100 steps (force + integrator) in one persistent launch",
                                  "value": inter * 100 / (med * 1e-3), "unit": "interactions/s",
                                  "ms_per_step": med / 100,
                                  "roofline": {"bound": "alu", "achieved": ach, "peak": fp32, "unit": "TFLOP/s",
                                               "frac": ach / fp32, "traffic": None}}
    del p4k, v4k

    # config 2: Black-Scholes 2^24 options: map (20 B/option) and fused map+reduce (12 B/option).
    # value = steady state (back-to-back launches alternating over two input/output sets, 2 x 201 MB
    # of inputs vs a 126-MB L2); the cold single launch (flushed L2) is reported beside it.
    n = 1 << 24
    sets = [tuple(torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=sd)) for sd in (2, 12)]
    S, X, T = sets[0]
    outs = [(torch.empty(n, dtype=torch.float32, device="cuda"), torch.empty(n, dtype=torch.float32, device="cuda"))
            for _ in sets]
    call, put = outs[0]
    cold, _ = time_launches(lambda: lime.map_blackscholes(S, X, T, inputs.BS_R, inputs.BS_SIGMA, call, put), 30, 5, flush,
                            writes_output=True)
    fns = [lambda k=k: lime.map_blackscholes(*sets[k], inputs.BS_R, inputs.BS_SIGMA, *outs[k]) for k in range(2)]
    med = time_back_to_back(fns, 20, 5, flush)
    gbs = 20.0 * n / (med * 1e-3) / 1e9
    out["blackscholes_map"] = {"workload": "configs[1]: Black-Scholes map, 2^24 options fp32", "value": n / (med * 1e-3),
                               "unit": "options/s", "ms_per_launch": med, "timing": "back-to-back, 2 input sets",
                               "ms_per_launch_cold": cold,
                               "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s", "frac": gbs / hbm,
                                            "frac_cold": 20.0 * n / (cold * 1e-3) / 1e9 / hbm,
                                            "traffic": ncu_traffic("bs_map")}}
    sums = [torch.empty(2, dtype=torch.float64, device="cuda") for _ in sets]
    cold, _ = time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, inputs.BS_R, inputs.BS_SIGMA, sums[0]),
                            30, 5, flush)
    fns = [lambda k=k: lime.map_reduce_blackscholes_sum(*sets[k], inputs.BS_R, inputs.BS_SIGMA, sums[k]) for k in range(2)]
    med = time_back_to_back(fns, 20, 5, flush)
    gbs = 12.0 * n / (med * 1e-3) / 1e9
    out["blackscholes_map_reduce"] = {"workload": "configs[1]: Black-Scholes fused map+reduce of total premium, 2^24 options",
                                      "value": n / (med * 1e-3), "unit": "options/s", "ms_per_launch": med,
                                      "timing": "back-to-back, 2 input sets", "ms_per_launch_cold": cold,
                                      "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s",
                                                   "frac": gbs / hbm, "frac_cold": 12.0 * n / (cold * 1e-3) / 1e9 / hbm,
                                                   "traffic": ncu_traffic("bs_map_reduce")}}
    del S, X, T, call, put, sets, outs, sums, fns

    # config 3: Mandelbrot 8192^2, max 1024 (11,856,987,162 iterations; 7 FP32 lane-ops each: x^2, y^2,
    # x^2 + y^2, x^2 - y^2, + cx, xy, fma(xy, 2, cy) -- the fewest exact ops of R7's recurrence)
    W = 8192
    d = 3.0 / W
    cnt = torch.empty((W, W), dtype=torch.int32, device="cuda")
    med, _ = time_launches(lambda: lime.map_mandelbrot(W, W, -2.0, -1.5, d, d, 1024, out=cnt), 10, 2, flush,
                           writes_output=True)
    iters = float(cnt.sum(dtype=torch.int64).item())
    lane_ops = 7.0 * iters / (med * 1e-3)
    peak_lane = SMS_B200 * 128 * SM_MAX_MHZ_NOMINAL * 1e6
    out["mandelbrot"] = {"workload": "configs[2]: Mandelbrot 8192x8192, max_iter 1024, int32 bit-exact",
                         "value": W * W / (med * 1e-3), "unit": "pixels/s", "iterations_per_s": iters / (med * 1e-3),
                         "ms_per_launch": med, "checksum": int(iters),
                         "roofline": {"bound": "alu", "achieved": lane_ops / 1e12, "peak": peak_lane / 1e12,
                                      "unit": "T FP32 lane-ops/s", "frac": lane_ops / peak_lane,
                                      "lane_ops_per_iteration": 7, "traffic": ncu_traffic("mandelbrot")}}
    del cnt

    # config 4: matmul 8192^3 bf16 -> fp32 (tcgen05)
    M = N = K = 8192
    try:
        A = torch.from_numpy(inputs.bf16_uniform(M, K, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
        Bt = torch.from_numpy(inputs.bf16_uniform(N, K, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
        Cm = torch.empty((M, N), dtype=torch.float32, device="cuda")
        med, _ = time_launches(lambda: lime.map_matmul_bf16(A, Bt, Cm), 20, 3, flush, writes_output=True)
        tf = 2.0 * M * N * K / (med * 1e-3) / 1e12
        cub, _ = time_launches(lambda: torch.matmul(A, Bt.t()), 20, 3, flush, writes_output=True)
        # cuBLAS with this kernel's own output type (fp32 C), the like-for-like library baseline
        cub32, _ = time_launches(lambda: torch.mm(A, Bt.t(), out_dtype=torch.float32), 20, 3, flush, writes_output=True)
        out["matmul"] = {"workload": "configs[3]: matmul 8192^3 bf16 in, fp32 accumulate/out (tcgen05)",
                         "value": M * N / (med * 1e-3), "unit": "dot products/s", "ms_per_launch": med,
                         "tflops": tf, "cublas_bf16_out_ms": cub, "cublas_fp32_out_ms": cub32,
                         "vs_cublas_fp32_out": cub32 / med,
                         "roofline": {"bound": "tensor", "achieved": tf, "peak": peaks["bf16_tflops"], "unit": "TFLOP/s",
                                      "frac": tf / peaks["bf16_tflops"], "traffic": ncu_traffic("matmul")}}
        del A, Bt, Cm
    except lime.LimeError as e:
        out["matmul"] = {"workload": "configs[3]", "unavailable": str(e)}

    # config 5 per-GPU shard at P = 8 (2^17 targets x 2^20 sources): the workload's equal masses take
    # the mass-factored element (11 FP32 lane-ops, R11); the same bodies with unequal
    # masses (U[0.5, 1.5)/N) take the per-body-mass element (12) -- both reported
    b1m = inputs.nbody_bodies(1 << 20, seed=5)
    b1m_mixed = b1m.copy()
    b1m_mixed[:, 3] = ((0.5 + inputs.uniform24(5, 99, 1 << 20)) / (1 << 20)).astype(np.float32)
    acc1m = torch.empty((1 << 17, 4), dtype=torch.float32, device="cuda")
    inter = float(1 << 20) * (1 << 17)
    for key, arr, ops in (("nbody_1m_p8_shard", b1m, FP32_LANE_OPS_UNIFORM_MASS),
                          ("nbody_1m_p8_shard_mixed_masses", b1m_mixed, FP32_LANE_OPS_PER_INTERACTION)):
        bd = torch.from_numpy(arr).cuda()
        med, _ = time_launches(lambda: lime.map_nbody(bd, EPS2, 0, 1 << 17, out=acc1m), 3, 1, flush)
        ach = FLOP_PER_INTERACTION * inter / (med * 1e-3) / 1e12
        out[key] = {"workload": "config-5 shard at P=8: 2^17 targets x 2^20 sources fp32"
                                + (", masses U[0.5,1.5)/N" if ops == FP32_LANE_OPS_PER_INTERACTION else ", equal masses"),
                    "value": inter / (med * 1e-3), "unit": "interactions/s", "ms_per_launch": med,
                    "fp32_lane_ops_per_interaction": ops,
                    "roofline": {"bound": "alu", "achieved": ach, "peak": fp32, "unit": "TFLOP/s", "frac": ach / fp32,
                                 "fp32_pipe_frac": ops * inter / (med * 1e-3) / (SMS_B200 * 128 * SM_MAX_MHZ_NOMINAL * 1e6),
                                 "traffic": ncu_traffic("nbody_force_1m_p8") if ops == FP32_LANE_OPS_UNIFORM_MASS else None}}
        del bd
    del acc1m
    # the headline's own size (2^20 x 2^20, one force launch) with the unequal masses: the number a
    # workload without the equal-mass fast path (R11) gets
    bd = torch.from_numpy(b1m_mixed).cuda()
    accm = torch.empty((1 << 20, 4), dtype=torch.float32, device="cuda")
    med, _ = time_launches(lambda: lime.map_nbody(bd, EPS2, out=accm), 2, 1, flush)
    inter_full = float(1 << 20) * (1 << 20)
    ach = FLOP_PER_INTERACTION * inter_full / (med * 1e-3) / 1e12
    out["nbody_1m_mixed_masses"] = {
        "workload": "configs[4] force map at full size (2^20 x 2^20 fp32), masses U[0.5,1.5)/N: per-body-mass element",
        "value": inter_full / (med * 1e-3), "unit": "interactions/s", "ms_per_launch": med,
        "fp32_lane_ops_per_interaction": FP32_LANE_OPS_PER_INTERACTION,
        "roofline": {"bound": "alu", "achieved": ach, "peak": fp32, "unit": "TFLOP/s", "frac": ach / fp32,
                     "fp32_pipe_frac": FP32_LANE_OPS_PER_INTERACTION * inter_full / (med * 1e-3)
                     / (SMS_B200 * 128 * SM_MAX_MHZ_NOMINAL * 1e6), "traffic": None}}
    del bd, accm

    # config-5 strong scaling on ONE GPU, compute only: the force map of the rank-0 shard at P = 1, 2, 4,
    # 8 (2^20/P targets x 2^20 sources, the launch each rank runs); E(P) = T_1 / (P T_P). The per-step
    # all-gather (2^20/P x 16 B out, 16 MiB in per rank) is what the driver's N-GPU runs add on top.
    bd = torch.from_numpy(b1m).cuda()
    acc_full = torch.empty((1 << 20, 4), dtype=torch.float32, device="cuda")
    shard_ms = {}
    for P in (1, 2, 4, 8):
        cnt = (1 << 20) // P
        shard_ms[P], _ = time_launches(lambda: lime.map_nbody(bd, EPS2, 0, cnt, out=acc_full[:cnt]), 3, 1, flush)
    out["nbody_1m_shard_scaling_probe"] = {
        "workload": "config-5 force map of one rank's shard at P = 1, 2, 4, 8 on one GPU (compute only)",
        "ms_per_launch": {str(P): v for P, v in shard_ms.items()},
        "compute_strong_scaling_efficiency": {str(P): shard_ms[1] / (P * v) for P, v in shard_ms.items()},
        "value": float(1 << 17) * (1 << 20) / (shard_ms[8] * 1e-3), "unit": "interactions/s (one P = 8 shard)",
        "projected_8gpu_interactions_per_s_compute_only": float(1 << 20) * (1 << 20) / (shard_ms[8] * 1e-3),
        "roofline": {"bound": "alu", "achieved": FLOP_PER_INTERACTION * float(1 << 17) * (1 << 20) / (shard_ms[8] * 1e-3) / 1e12,
                     "peak": fp32, "unit": "TFLOP/s",
                     "frac": FLOP_PER_INTERACTION * float(1 << 17) * (1 << 20) / (shard_ms[8] * 1e-3) / 1e12 / fp32,
                     "traffic": None}}
    del bd, acc_full

    # F3: double-precision N-Body (Table 3) at the config-5 per-GPU shape of P = 8; FP64-pipe
    # bound: 16 FP64 ops per interaction at 64 lanes/clk/SM (microbench: 58.9 measured)
    b64 = torch.from_numpy(inputs.nbody_bodies(1 << 20, seed=5).astype(np.float64)).cuda()
    acc64 = torch.empty((1 << 17, 4), dtype=torch.float64, device="cuda")
    med, _ = time_launches(lambda: lime.map_nbody_f64(b64, EPS2, 0, 1 << 17, out=acc64), 3, 1, flush)
    inter = float(1 << 20) * (1 << 17)
    fp64_peak = 64.0 * SMS_B200 * SM_MAX_MHZ_NOMINAL * 1e6
    out["nbody_f64"] = {"workload": "F3: N-body fp64, 2^17 targets x 2^20 sources (config-5 shard at P=8)",
                        "value": inter / (med * 1e-3), "unit": "interactions/s", "ms_per_launch": med,
                        "roofline": {"bound": "alu", "achieved": 16 * inter / (med * 1e-3) / 1e12,
                                     "peak": fp64_peak / 1e12, "unit": "T FP64 lane-ops/s",
                                     "frac": 16 * inter / (med * 1e-3) / fp64_peak, "traffic": ncu_traffic("nbody_f64")}}
    del b64, acc64

    # F2: Parboil-CP and MRI-Q at the paper's Table 3 sizes (L353-354); both are
    # bound by the MUFU (XU) pipe: 1 rsqrt (CP) / 1 sin + 1 cos (MRI-Q) per interaction.
    mufu_peak = 16.0 * SMS_B200 * SM_MAX_MHZ_NOMINAL * 1e6      # 16 lanes/clk/SM (microbench: 16.00)
    atoms = torch.from_numpy(inputs.cp_atoms()).cuda()
    npts = inputs.CP_NX * inputs.CP_NY
    V = torch.empty(npts, device="cuda")
    med, _ = time_launches(lambda: lime.map_coulomb(atoms, inputs.CP_NX, inputs.CP_NY, inputs.CP_Z, inputs.CP_H, out=V),
                           30, 3, flush)
    inter = float(npts) * atoms.shape[0]
    out["parboil_cp"] = {"workload": "F2: Parboil-CP Coulombic potential, 3968 atoms x 512^2 lattice (Table 3)",
                         "value": inter / (med * 1e-3), "unit": "interactions/s", "ms_per_launch": med,
                         "roofline": {"bound": "alu", "achieved": inter / (med * 1e-3) / 1e12, "peak": mufu_peak / 1e12,
                                      "unit": "T MUFU ops/s", "frac": inter / (med * 1e-3) / mufu_peak,
                                      "traffic": ncu_traffic("parboil_cp")}}
    k = torch.from_numpy(inputs.mriq_kspace()).cuda()
    vx = torch.from_numpy(inputs.mriq_voxels()).cuda()
    Q = torch.empty((vx.shape[0], 2), device="cuda")
    med, _ = time_launches(lambda: lime.map_mriq(k, vx, out=Q), 30, 3, flush)
    inter = float(vx.shape[0]) * k.shape[0]
    out["parboil_mriq"] = {"workload": "F2: Parboil-MRI-Q, 3072 k-samples x 32768 voxels (Table 3)",
                           "value": inter / (med * 1e-3), "unit": "interactions/s", "ms_per_launch": med,
                           "roofline": {"bound": "alu", "achieved": 2 * inter / (med * 1e-3) / 1e12,
                                        "peak": mufu_peak / 1e12, "unit": "T MUFU ops/s",
                                        "frac": 2 * inter / (med * 1e-3) / mufu_peak, "traffic": ncu_traffic("parboil_mriq")}}
    del atoms, V, k, vx, Q

    # F4: JG-Series (100,000 coefficient pairs, Table 3) and JG-Crypt (IDEA over 3 MiB, L354-355)
    fp32_lane_peak = 128.0 * SMS_B200 * SM_MAX_MHZ_NOMINAL * 1e6
    for dt, nm in ((torch.float32, "jg_series_f32"), (torch.float64, "jg_series_f64")):
        so = torch.empty((inputs.SERIES_N, 2), dtype=dt, device="cuda")
        med, _ = time_launches(lambda: lime.map_series(0, inputs.SERIES_N, dtype=dt, out=so), 20, 3, flush)
        terms = float(inputs.SERIES_N) * 1001
        # algorithmic work: one complex multiply-add g_i * e^{i theta n i} per term = 2 FMA lane-ops
        peak = fp32_lane_peak if dt == torch.float32 else fp64_peak
        ach = 2 * terms / (med * 1e-3)
        out[nm] = {"workload": f"F4: JG-Series {'fp32' if dt == torch.float32 else 'fp64'}, 100,000 coefficient pairs x 1001 nodes",
                   "value": inputs.SERIES_N / (med * 1e-3), "unit": "coefficient pairs/s", "ms_per_launch": med,
                   "terms_per_s": terms / (med * 1e-3),
                   "roofline": {"bound": "alu", "achieved": ach / 1e12, "peak": peak / 1e12,
                                "unit": "T FP32 lane-ops/s" if dt == torch.float32 else "T FP64 lane-ops/s",
                                "frac": ach / peak, "traffic": None}}
        del so
    data = torch.from_numpy(inputs.crypt_data()).cuda()
    ek, _ = lime.idea_key_schedule(inputs.crypt_key())
    enc = torch.empty_like(data)
    med, _ = time_launches(lambda: lime.map_idea(data, ek, out=enc), 30, 3, flush)
    # integer-issue roofline: the IDEA round function is multiplications mod
    # 2^16+1, additions and XORs on the ALU/FMA(IMAD) pipes; the bound is instruction issue, one
    # warp-instruction per SMSP per clock = 148 x 4 x 32 thread-instructions/clk. The kernel's
    # loop runs IDEA_SASS_PER_UNIT SASS instructions per 16-byte unit (two 8-byte blocks; counted
    # from cuobjdump, pinned by tests/test_sass_guards.py).
    units = data.numel() / 16.0
    issue_peak = SMS_B200 * 4 * 32 * SM_MAX_MHZ_NOMINAL * 1e6
    ach = units * IDEA_SASS_PER_UNIT / (med * 1e-3)
    out["jg_crypt"] = {"workload": "F4: JG-Crypt IDEA-ECB over 3 MiB (Table 3)", "value": data.numel() / (med * 1e-3),
                       "unit": "bytes/s", "ms_per_launch": med, "hbm_GBs": 2.0 * data.numel() / (med * 1e-3) / 1e9,
                       "roofline": {"bound": "issue", "achieved": ach / 1e12, "peak": issue_peak / 1e12,
                                    "unit": "T thread-instructions/s", "frac": ach / issue_peak, "traffic": None,
                                    "sass_per_16B_unit": IDEA_SASS_PER_UNIT,
                                    "note": "one wave of CTAs over 3 MiB: the issue-bound work is ~3.5 us at 1965 MHz, so "
                                            "launch/ramp (~5-6 us of the event-timed launch, tools/launch_floor.py) "
                                            "dominates; HBM traffic (6 MB) is 1 us at HBM speed"}}
    del data, enc

    # reduction `!`: sum over 2^28 fp32 (1 GiB)
    x = torch.ones(1 << 28, dtype=torch.float32, device="cuda")
    r = torch.empty((), dtype=torch.float32, device="cuda")
    med, _ = time_launches(lambda: lime.reduce_sum(x, r), 20, 3, flush)
    gbs = 4.0 * (1 << 28) / (med * 1e-3) / 1e9
    out["reduce_sum_f32"] = {"workload": "reduce ! sum over 2^28 fp32", "value": (1 << 28) / (med * 1e-3),
                             "unit": "elements/s", "ms_per_launch": med,
                             "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s", "frac": gbs / hbm,
                                          "traffic": ncu_traffic("reduce_sum_f32")}}
    del x
    return out


# ----------------------------------------------------------------------------- sharded configs (any N)
def run_sharded(args, rank, world, local, peaks, flush):
    """Configs 2-4 partitioned over the N ranks exactly as SURVEY.md §8(e) says, at every N (so the
    driver's N = 1, 2, 4, 8 runs each report every config): Black-Scholes fused map+reduce over
    contiguous option shards + one all_reduce of the fp64 partials (strong: one 2^24 array; weak:
    2^24 options per GPU), Mandelbrot 8192^2 over cyclic rows, matmul 8192^3 over C row blocks (Bt
    replicated before timing). Per rank: warm-up, then each launch between CUDA events on the
    launching stream after an L2 flush; value = all ranks' units / the MAX over ranks of the median
    launch time."""
    hbm = peaks["hbm_gbs"]
    out = {}

    def timed(fn, reps, warm, writes_output=False):
        barrier(world)
        med, _ = time_launches(fn, reps, warm, flush, writes_output=writes_output)
        return max_over_ranks(med, world)

    n = 1 << 24
    S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
    b, c = ldist.shard_range_aligned(n, rank, world, 4)
    ms = timed(lambda: ldist.blackscholes_shard_total(S, X, T, inputs.BS_R, inputs.BS_SIGMA), 30, 5)
    gbs = 12.0 * n / (ms * 1e-3) / 1e9 / world          # per-GPU HBM rate
    out["blackscholes_map_reduce_strong"] = {
        "workload": f"configs[1]: fused Black-Scholes total premium, 2^24 options split over {world} GPU(s) "
                    "(contiguous shards) + all_reduce of 2 fp64 partials", "scaling": "strong",
        "value": n / (ms * 1e-3), "unit": "options/s", "ms_per_call": ms, "options_per_gpu": c,
        "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s per GPU", "frac": gbs / hbm}}
    del S, X, T
    Sw, Xw, Tw = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=200 + rank))
    ms = timed(lambda: ldist.blackscholes_total(Sw, Xw, Tw, inputs.BS_R, inputs.BS_SIGMA), 30, 5)
    gbs = 12.0 * n / (ms * 1e-3) / 1e9
    out["blackscholes_map_reduce_weak"] = {
        "workload": "configs[1] weak scaling: fused Black-Scholes total premium, 2^24 options PER GPU "
                    "+ all_reduce of 2 fp64 partials", "scaling": "weak",
        "value": float(n) * world / (ms * 1e-3), "unit": "options/s", "ms_per_call": ms,
        "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s per GPU", "frac": gbs / hbm}}
    del Sw, Xw, Tw

    W = 8192
    d = 3.0 / W
    first, stride, rows = ldist.cyclic_rows(W, rank, world)
    cnt = torch.empty((rows, W), dtype=torch.int32, device="cuda")
    ms = timed(lambda: ldist.mandelbrot_cyclic(W, W, -2.0, -1.5, d, d, 1024, out=cnt), 10, 2, writes_output=True)
    iters = torch.tensor([float(cnt.sum(dtype=torch.int64).item())], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(iters)
    lane_peak = SMS_B200 * 128 * SM_MAX_MHZ_NOMINAL * 1e6
    out["mandelbrot_cyclic_rows"] = {
        "workload": f"configs[2]: Mandelbrot 8192x8192, max_iter 1024, cyclic rows over {world} GPU(s)",
        "scaling": "strong", "value": W * W / (ms * 1e-3), "unit": "pixels/s", "ms_per_call": ms,
        "rows_per_gpu": rows, "checksum": int(iters.item()),
        "roofline": {"bound": "alu", "achieved": 7.0 * iters.item() / world / (ms * 1e-3) / 1e12,
                     "peak": lane_peak / 1e12, "unit": "T FP32 lane-ops/s per GPU",
                     "frac": 7.0 * iters.item() / world / (ms * 1e-3) / lane_peak}}
    del cnt

    M = N = K = 8192
    try:
        A = torch.from_numpy(inputs.bf16_uniform(M, K, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
        Bt = torch.from_numpy(inputs.bf16_uniform(N, K, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
        mb, mc = ldist.shard_range(M, rank, world)
        Cb = torch.empty((mc, N), dtype=torch.float32, device="cuda")
        ms = timed(lambda: ldist.matmul_row_block(A, Bt, Cb), 20, 3, writes_output=True)
        tf = 2.0 * mc * N * K / (ms * 1e-3) / 1e12
        out["matmul_row_blocks"] = {
            "workload": f"configs[3]: matmul 8192^3 bf16 -> fp32, C row blocks over {world} GPU(s), Bt replicated",
            "scaling": "strong", "value": M * N / (ms * 1e-3), "unit": "dot products/s", "ms_per_call": ms,
            "rows_per_gpu": mc,
            "roofline": {"bound": "tensor", "achieved": tf, "peak": peaks["bf16_tflops"], "unit": "TFLOP/s per GPU",
                         "frac": tf / peaks["bf16_tflops"]}}
        del A, Bt, Cb
    except lime.LimeError as e:
        out["matmul_row_blocks"] = {"workload": "configs[3]", "unavailable": str(e)}
    return out


# ----------------------------------------------------------------------------- CPU oracle
def cpu_oracle_sample(n: int, targets: int):
    """The oracle as it stands (single-threaded C, fp64): accelerations of `targets` targets
    against all n sources of the same workload. Returns (interactions/s, seconds)."""
    import oracle
    b = inputs.nbody_bodies(n, seed=5)
    oracle.lib()
    t = time.perf_counter()
    oracle.nbody_accel(b, np.float32(EPS2), 0, targets)
    dt = time.perf_counter() - t
    return targets * float(n) / dt, dt


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class one_core:
    """Pin this process to one host core while the oracle is timed (the oracle
    beside the GPU runs single-threaded on one pinned core)."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0) if hasattr(os, "sched_getaffinity") else None
        if self.old:
            os.sched_setaffinity(0, {min(self.old)})
        return self

    def __exit__(self, *exc):
        if self.old:
            os.sched_setaffinity(0, self.old)


def oracle_beside(configs: dict) -> None:
    """Time the oracle (as it stands, one pinned core) on a bounded sample of every config's
    workload and attach it as configs[k]["cpu_oracle"] in the config's own unit."""
    import oracle
    oracle.lib()

    def timed(fn):
        t = time.perf_counter()
        r = fn()
        return r, time.perf_counter() - t

    def put(key, units, secs, sample):
        if key in configs and isinstance(configs[key], dict):
            configs[key]["cpu_oracle"] = {"value": units / secs, "unit": configs[key].get("unit"), "cores": 1,
                                          "kind": "oracle", "sample": f"{sample} ({secs:.2f} s)"}

    with one_core():
        b = inputs.nbody_bodies(4096, seed=1)
        _, sec = timed(lambda: oracle.nbody_accel(b, np.float32(EPS2)))
        put("nbody_4096", 4096.0 * 4096, sec, "full 4096 x 4096 force map")
        put("nbody_4096_graph", 4096.0 * 4096, sec, "one 4096 x 4096 force map (integrator negligible)")
        put("nbody_4096_simulate", 4096.0 * 4096, sec, "one 4096 x 4096 force map (integrator negligible)")
        S, X, T = inputs.blackscholes_options(1 << 20, seed=2)
        _, sec = timed(lambda: oracle.blackscholes(S, X, T, inputs.BS_R, inputs.BS_SIGMA))
        put("blackscholes_map", float(1 << 20), sec, "2^20 of the 2^24 options")
        _, sec = timed(lambda: oracle.blackscholes_sums(S, X, T, inputs.BS_R, inputs.BS_SIGMA))
        put("blackscholes_map_reduce", float(1 << 20), sec, "2^20 of the 2^24 options")
        W = 8192
        rows = 64
        _, sec = timed(lambda: oracle.mandelbrot(W, W, 0, W // rows, rows, -2.0, -1.5, 3.0 / W, 3.0 / W, 1024))
        put("mandelbrot", float(rows * W), sec, f"{rows} rows spread evenly over the 8192^2 frame")
        A = inputs.bf16_uniform(64, 8192, 4, 0)
        Bt = inputs.bf16_uniform(64, 8192, 4, 1)
        rr = np.random.default_rng(0).integers(0, 64, size=(2, 8192))
        _, sec = timed(lambda: oracle.matmul_bf16_entries(A, Bt, rr[0], rr[1]))
        put("matmul", 8192.0, sec, "8192 dot products of length K = 8192")
        b64 = inputs.nbody_bodies(1 << 20, seed=5).astype(np.float64)
        _, sec = timed(lambda: oracle.nbody_accel_f64(b64, 1e-4, 0, 32))
        put("nbody_f64", 32.0 * (1 << 20), sec, "32 targets x 2^20 sources")
        atoms = inputs.cp_atoms()
        _, sec = timed(lambda: oracle.coulomb_potential(atoms, inputs.CP_NX, 8, inputs.CP_Z, inputs.CP_H))
        put("parboil_cp", 8.0 * inputs.CP_NX * atoms.shape[0], sec, "8 lattice rows x all atoms")
        ks, vx = inputs.mriq_kspace(), inputs.mriq_voxels()
        _, sec = timed(lambda: oracle.mriq(ks, vx[:2048]))
        put("parboil_mriq", 2048.0 * ks.shape[0], sec, "2048 voxels x all k-samples")
        _, sec = timed(lambda: oracle.series(0, 1000))
        put("jg_series_f32", 1000.0, sec, "coefficients 0..999")
        put("jg_series_f64", 1000.0, sec, "coefficients 0..999")
        data = inputs.crypt_data()
        ek, _ = oracle.idea_keys(inputs.crypt_key())
        _, sec = timed(lambda: oracle.idea(data, ek))
        put("jg_crypt", float(data.shape[0]), sec, "the full 3 MiB")
        x = np.ones(1 << 26, dtype=np.float32)
        _, sec = timed(lambda: oracle.reduce("sum", x, "f32"))
        put("reduce_sum_f32", float(1 << 26), sec, "2^26 of the 2^28 elements")


def headline_config(n, world):
    """The headline workload's config, shared by both arms (the reference arm times a bounded oracle
    sample of this same workload, described in its cpu_baseline.sample)."""
    return {"workload": f"BASELINE.json configs[4]: N-body all-pairs {n} bodies fp32, index-space "
                        "sharded, NCCL all-gather per step",
            "n_bodies": n, "eps2": EPS2, "dt": DT, "targets_per_gpu": n // world,
            "parallelism": f"target-index shards x{world}" + (" + all_gather" if world > 1 else ""),
            "l2": "flushed before every step inside the timed region (2x L2 write); the 16 MiB source "
                  "array is then re-read from L2 by design (broadcast operand)",
            "inputs": "inputs.nbody_bodies(seed=5): U[-1,1)^3, m=1/N, v0=0"}


def run_reference(args, rank, world):
    if rank != 0:
        return None
    import oracle
    n = args.n
    b = inputs.nbody_bodies(n, seed=5)
    vel = np.zeros((args.ref_targets, 4), dtype=np.float32)
    oracle.lib()
    times = []
    for k in range(args.warmup + args.steps):
        t = time.perf_counter()
        lo = (k * args.ref_targets) % n
        acc = oracle.nbody_accel(b, np.float32(EPS2), lo, args.ref_targets)
        a4 = np.zeros((args.ref_targets, 4), dtype=np.float32)
        a4[:, :3] = acc
        oracle.nbody_integrate(b[lo:lo + args.ref_targets], vel, a4, np.float32(DT))
        if k >= args.warmup:
            times.append(time.perf_counter() - t)
    per_step = float(np.mean(times))
    value = args.ref_targets * float(n) / per_step
    sample = f"{args.ref_targets} targets x {n} sources (+ integrator) of the config-5 workload per step"
    return {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": per_step * 1e3, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": headline_config(n, world),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


# ----------------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["lime", "reference"], default="lime")
    ap.add_argument("--bodies", dest="n", type=int, default=1 << 20)
    ap.add_argument("--no-extras", action="store_true", help="skip the N = 1 per-config extras")
    ap.add_argument("--no-sharded", action="store_true", help="skip the sharded configs 2-4 (any N)")
    ap.add_argument("--cpu-targets", type=int, default=3072)
    ap.add_argument("--ref-targets", type=int, default=512)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "lime" else args.warmup

    rank, world, local = dist_init(args)
    if args.impl == "reference":
        line = run_reference(args, rank, world)
        if line is not None:
            print(json.dumps(line), flush=True)
        return

    lime.load()
    peaks = measured_peaks()
    line = run_nbody(args, rank, world, local)
    if not args.no_sharded:
        props = torch.cuda.get_device_properties(local)
        flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
        if world == 1:
            try:      # a failing sub-config must not cost the headline line (world 1: no collectives to strand)
                sharded = run_sharded(args, rank, world, local, peaks, flush)
            except Exception as e:  # noqa: BLE001
                sharded = {"error": f"{type(e).__name__}: {e}"}
        else:
            sharded = run_sharded(args, rank, world, local, peaks, flush)
        del flush
        if rank == 0:
            line["sharded_configs"] = sharded
    if rank == 0 and world == 1:
        if not args.no_extras:
            props = torch.cuda.get_device_properties(local)
            flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
            try:
                line["configs"] = run_extras(peaks, flush)
            except Exception as e:  # noqa: BLE001
                line["configs"] = {"error": f"{type(e).__name__}: {e}"}
            line["configs_timing"] = ("per config: warm-up launches, then each timed launch preceded (outside the "
                                      "CUDA-event pair) by an L2 flush and a ~100-us device sleep so the launch is "
                                      "queued before the start event; median over launches. Flush = write of 2x L2 "
                                      "(L2 left full of dirty lines) for kernels whose output exceeds L2 "
                                      "(Black-Scholes map, Mandelbrot, matmul + cuBLAS), else that write followed by "
                                      "a read of another 2x L2 buffer (clean L2): the L2 state the same kernel "
                                      "leaves behind when run back to back")
            try:
                oracle_beside(line["configs"])
            except Exception as e:  # noqa: BLE001
                line["configs_oracle_error"] = f"{type(e).__name__}: {e}"
        with one_core():
            v, secs = cpu_oracle_sample(args.n, args.cpu_targets)
        line["cpu_baseline"] = {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
                                "sample": f"{args.cpu_targets} targets x {args.n} sources of step 0 "
                                          f"({secs:.1f} s, single-threaded C fp64, one pinned core)",
                                "host_cpu": cpu_model(), "host_cores": os.cpu_count()}
    elif rank == 0:
        line["cpu_baseline"] = None
    line["peaks"] = peaks
    # compact digest of every sub-line, LAST in the JSON line so that a driver keeping only the tail
    # of stdout still sees each config's time and roofline fraction
    digest = {}
    for group in ("configs", "sharded_configs"):
        for k, v in (line.get(group) or {}).items():
            if isinstance(v, dict) and "roofline" in v:
                t = v.get("ms_per_launch", v.get("ms_per_step", v.get("ms_per_call")))
                digest[k] = {"ms": t if not isinstance(t, dict) else None, "value": v.get("value"),
                             "unit": v.get("unit"), "frac": v["roofline"].get("frac"),
                             "bound": v["roofline"].get("bound")}
    line["digest"] = digest
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
