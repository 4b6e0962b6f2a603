#!/usr/bin/env python
"""bench.py — the driver's benchmark contract for the PolyHankel forward
convolution on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload conv3x] [--math bf16|tf32|fp32]

A "step" is one pass of the whole hot path (pack ->
coefficient MAC over channels -> extraction/NCHW store) over one batch of
synthetic input, through the C-ABI (polyconv_forward).  Workload at N=1 is
BASELINE.json configs[1], the ResNet-50 conv3_x layer (N=32, C=K=128, 28x28,
3x3, pad 1), BF16 in/out and BF16 tensor-core math.  Metric: effective
TFLOP/s = 2*N*K*C*R*S*P*Q / t (BASELINE.json metric, north_star FLOP formula).

Timing: W untimed warm-up steps; K timed steps, each
bracketed by CUDA events on the launching stream, L2 flushed between steps by
a 256 MiB write (inputs are 6.4 MB and would otherwise sit in the 126 MB L2)
followed by a 256 MiB read, so that the flush's dirty lines are written back
before the step instead of inside it;
barrier + synchronize around the timed region; max over ranks.  The dominant
kernel (the MAC) is timed live with events the library records around its
launch (polyconv_plan_set_timing_events).  Clocks and throttle reasons are
sampled through NVML during the timed region.

Multi-GPU (torchrun, one process per GPU): weak scaling by batch -- every rank
runs its own N=32 batch (images are independent, Eq. 12 per item, P.1398);
there is no data-path collective.  value = FLOPs of all ranks / max-rank time.

--impl reference: the fp64 CPU oracle (oracle/, the test oracle, untuned) on
the host cores, rank 0 only, each step a bounded sample of the same workload
(a subset of (image, output-channel) planes) so the whole run ends in minutes.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

METRIC = "conv fwd effective TFLOP/s and % roofline per layer at 1/2/4/8 B200 vs cuDNN"
UNIT = "TFLOP/s"
WORKLOADS = {"conv3x": synth.CONV3X, "resnet50": None}   # resnet50: BASELINE configs[4], strong scaling
L2_FLUSH_BYTES = 256 << 20
PROFILES = os.path.join(ROOT, "profiles")


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except (OSError, ValueError):
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


def _roofline_peak(math, peaks):
    """Peak of the contraction's own dtype (B200_PROFILING.md: another dtype's
    measured peak x the nominal ratio).  bf16: measured burst; tf32: measured
    bf16 x 1.1/2.25; fp32 FFMA: 'alu' peak 148 SM x 128 lanes x 2 x 1.965 GHz."""
    if math == "bf16":
        return "tensor", peaks["bf16_tflops"], "bf16_tflops (burst) of MEASURED_PEAKS.json"
    if math == "tf32":
        return "tensor", peaks["bf16_tflops"] * 1.1 / 2.25, "bf16_tflops x 1.1/2.25 (nominal tf32:bf16)"
    return "alu", 148 * 128 * 2 * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6 / 1e12, \
        "148 SM x 128 FP32 lanes x 2 FLOP x sm_max_mhz"


def _traffic(kernel_key, field="dram"):
    """Bytes per launch of the dominant kernel from the committed ncu --set full summary
    (profiles/ncu_summary.json), else None.  field "dram": dram read + write; "l2_write": the
    bytes the kernel writes into L2 (32-byte sectors) -- the output y stays dirty in L2 when
    the kernel ends, so its DRAM write-back is not in the kernel's own dram counters."""
    try:
        with open(os.path.join(PROFILES, "ncu_summary.json")) as f:
            d = json.load(f)
        e = d.get(kernel_key)
        if not e:
            return None
        if field == "l2_write":
            return int(e["l2_write_sectors"] * 32)
        return int(e["dram_bytes_read"] + e["dram_bytes_write"])
    except (OSError, ValueError, KeyError, TypeError):
        return None


class ClockSampler:
    """NVML polling thread: SM clock and clock-event reasons while running."""

    REASONS = [("gpu_idle", "nvmlClocksEventReasonGpuIdle"),
               ("applications_clocks_setting", "nvmlClocksEventReasonApplicationsClocksSetting"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
               ("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("sync_boost", "nvmlClocksEventReasonSyncBoost"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("hw_power_brake_slowdown", "nvmlClocksEventReasonHwPowerBrakeSlowdown")]

    def __init__(self, device_index, period_s=0.002):
        self.ok = False
        self.samples = []
        self.reasons = set()
        self.period = period_s
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            uuid = None
            try:
                import torch
                uuid = str(torch.cuda.get_device_properties(device_index).uuid)
            except Exception:
                pass
            h = None
            if uuid:
                for i in range(pynvml.nvmlDeviceGetCount()):
                    hh = pynvml.nvmlDeviceGetHandleByIndex(i)
                    u = pynvml.nvmlDeviceGetUUID(hh)
                    u = u.decode() if isinstance(u, bytes) else u
                    if u.replace("GPU-", "") == uuid.replace("GPU-", ""):
                        h = hh
            self.h = h if h is not None else pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # no NVML: report it instead of guessing
            self.err = str(e)

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                mhz = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append(mhz)
                for name, attr in self.REASONS:
                    if r & getattr(nv, attr, 0):
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "note": "NVML unavailable: %s" % self.err}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons - {"gpu_idle"}), "samples": len(self.samples)}


# ----------------------------------------------------------------- reference arm --

def run_reference(args, rank, world):
    """The oracle (fp64 CPU direct convolution, untuned) as the reference arm."""
    if rank != 0:
        return 0
    import oracle
    # resnet50 (strong scaling): the oracle samples its l2 3x3 layer
    shape = WORKLOADS[args.workload] or next(L for L in synth.RESNET50 if L.name == "l2_3x3_128")
    x, w = synth.make_inputs(shape, synth.seed_for(1), "uniform", batch=(0, 1))
    cores = oracle.max_threads()
    # calibrate: one image, all K output planes
    t0 = time.perf_counter()
    oracle.conv2d(x, w, shape.stride, shape.padding)
    per_plane = (time.perf_counter() - t0) / shape.K
    budget = float(os.environ.get("POLYCONV_REF_BUDGET_S", "90"))
    planes = int(max(1, min(shape.K, budget / max(1, args.steps + args.warmup) / max(per_plane, 1e-9))))
    ws = w[:planes]
    flop = 2 * planes * shape.C * shape.R * shape.S * shape.P * shape.Q
    for _ in range(args.warmup):
        oracle.conv2d(x, ws, shape.stride, shape.padding)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.conv2d(x, ws, shape.stride, shape.padding)
        ts.append(time.perf_counter() - t0)
    t = sum(ts)
    value = flop * args.steps / t / 1e12
    sample = "image 0 of %s, %d of %d output-channel planes per step (%.3g GFLOP/step)" % (
        shape.name, planes, shape.K, flop / 1e9)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": shape.name, "N": shape.N, "C": shape.C, "K": shape.K, "H": shape.H,
                       "W": shape.W, "R": shape.R, "S": shape.S, "stride": list(shape.stride),
                       "padding": list(shape.padding), "sample": sample},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "gpu_launches": 0}
    print(json.dumps(line), flush=True)
    return 0



# ------------------------------------------------------- config 4: strong scaling --

def run_resnet50(args, torch, dist, pc, dev, rank, world, local):
    """BASELINE configs[4]: all 53 forward convs of ResNet-50 v1.5 at N=256 (23 unique shapes,
    synth.RESNET50 with counts), the batch split over the ranks (images [r*N/G, (r+1)*N/G)),
    filters replicated; one step = every conv once on this rank's shard, L2 flushed before the
    step.  value = FLOPs of the whole N=256 stack / max-rank step time (strong scaling)."""
    io = "bf16" if args.math == "bf16" else "f32"
    tdt = torch.bfloat16 if io == "bf16" else torch.float32
    N = 256
    lo, hi = N * rank // world, N * (rank + 1) // world
    nb = hi - lo
    layers = []
    for li, L in enumerate(synth.RESNET50):
        g = torch.Generator(device=dev).manual_seed(synth.seed_for(4, li) + rank)
        x = (torch.rand((nb, L.C, L.H, L.W), device=dev, generator=g) * 2 - 1).to(tdt)
        w = ((torch.rand((L.K, L.C, L.R, L.S), device=dev, generator=g) * 2 - 1) / (L.C * L.R * L.S) ** 0.5).to(tdt)
        plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math=args.math, io_dtype=io, device=local)
        y = torch.empty(plan.output_shape, dtype=tdt, device=dev)
        layers.append((L, plan, x, w, y))
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)

    def step():
        for L, plan, x, w, y in layers:
            for _ in range(L.count):
                plan.forward(x, w, y)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        flush.zero_()
        step()
    barrier()
    stream = torch.cuda.current_stream()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    sampler = ClockSampler(local)
    with sampler:
        barrier()
        for a, b in ev:
            flush.zero_()
            a.record(stream)
            step()
            b.record(stream)
        barrier()
    t = torch.tensor([sum(a.elapsed_time(b) for a, b in ev) / args.steps], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    F = sum(L.count * L.flops() for L in synth.RESNET50)   # whole N=256 stack
    value = F / (float(t) * 1e-3) / 1e12
    # end to end: the same step through polyconv_forward_host with pinned host buffers (one
    # step: 11 GB of activations cross PCIe per pass, so a single timed pass)
    hosts = [(L, plan, x.cpu().pin_memory(), w.cpu().pin_memory(),
              torch.empty(plan.output_shape, dtype=tdt).pin_memory()) for L, plan, x, w, y in layers]
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    h2d = d2h = 0
    for L, plan, xh, wh, yh in hosts:
        for _ in range(L.count):
            plan.forward_host(xh, wh, yh)
            h2d += xh.numel() * xh.element_size() + wh.numel() * wh.element_size()
            d2h += yh.numel() * yh.element_size()
    e1.record(stream)
    barrier()
    te = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    kernels = {}
    for L, plan, *_ in layers:
        k = plan.info()["kernel"]
        kernels[k] = kernels.get(k, 0) + L.count
    launches = sum(L.count * plan.info()["launches"] for L, plan, *_ in layers) * args.steps
    if rank == 0:
        peaks, src = _peaks()
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": float(t), "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": args.math, "data": "synthetic",
                "config": {"workload": "resnet50_n256_forward_convs", "N": N, "per_rank_batch": nb,
                           "convs": sum(L.count for L in synth.RESNET50), "unique_shapes": len(synth.RESNET50),
                           "io_dtype": io, "math": args.math, "kernels": kernels,
                           "parallelism": "batch-sharded x%d (strong: N=256 split, no collective)" % world,
                           "l2": "flushed before every step (256 MiB write)"},
                "e2e": {"value": F / (float(te) * 1e-3) / 1e12, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                        "d2h_bytes_per_step": int(d2h), "ms_per_step": float(te), "api": "polyconv_forward_host"},
                "gpu_launches": int(launches), "clocks": sampler.summary(),
                "roofline": {"bound": "tensor", "peak": peaks["bf16_tflops"], "unit": "TFLOP/s",
                             "achieved": value / world, "frac": value / world / peaks["bf16_tflops"],
                             "traffic": None, "note": "whole stack per GPU against the bf16 peak (%s)" % src}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0

def cpu_baseline(shape):
    """Oracle timed on the host cores on a bounded sample (~10-20 s of CPU work)."""
    import oracle
    x1, w = synth.make_inputs(shape, synth.seed_for(1), "uniform", batch=(0, 1))
    t0 = time.perf_counter()
    oracle.conv2d(x1, w, shape.stride, shape.padding)
    t1 = time.perf_counter() - t0
    target = float(os.environ.get("POLYCONV_CPU_BASELINE_S", "12"))
    n = int(max(1, min(shape.N, target / max(t1, 1e-6))))
    x, _ = synth.make_inputs(shape, synth.seed_for(1), "uniform", batch=(0, n))
    t0 = time.perf_counter()
    oracle.conv2d(x, w, shape.stride, shape.padding)
    t = time.perf_counter() - t0
    flop = shape.with_batch(n).flops()
    return {"value": flop / t / 1e12, "unit": UNIT, "cores": oracle.max_threads(), "kind": "oracle",
            "sample": "%d of %d images of %s (%.2f GFLOP, %.1f s)" % (n, shape.N, shape.name, flop / 1e9, t)}


# ----------------------------------------------------------------------- our arm --

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="conv3x", choices=sorted(WORKLOADS),
                    help="conv3x: configs[1], weak scaling by batch; resnet50: configs[4], the 53 forward "
                         "convs of ResNet-50 at N=256 split over the ranks (strong scaling)")
    ap.add_argument("--math", default="bf16", choices=["bf16", "tf32", "fp32"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cudnn", action="store_true")
    ap.add_argument("--kernel", default="auto", help="force a MAC variant (ablation; default auto)")
    ap.add_argument("--no-gate", action="store_true", help="skip the ResNet-50 N=256 3x3 gate records")
    ap.add_argument("--no-by-math", action="store_true", help="skip the TF32 / FP32 conv3x records")
    args = ap.parse_args()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # one process per GPU: re-launch this command under torch.distributed.run
        import subprocess
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(args.gpus),
               "--master-addr", "127.0.0.1", "--master-port", os.environ.get("MASTER_PORT", "29531"),
               os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd)
    if world != args.gpus:
        raise SystemExit("--gpus %d but WORLD_SIZE=%d: launch one process per GPU" % (args.gpus, world))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")

    import torch
    import torch.distributed as dist
    import paper_conf_cgo_xuzc025_b200 as pc

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    if args.workload == "resnet50":
        return run_resnet50(args, torch, dist, pc, dev, rank, world, local)
    shape = WORKLOADS[args.workload]
    io = "bf16" if args.math == "bf16" else "f32"
    tdt = torch.bfloat16 if io == "bf16" else torch.float32
    eb = 2 if io == "bf16" else 4

    # seeded synthetic inputs (per-rank images: weak scaling by batch)
    x_np, w_np = synth.make_inputs(shape, synth.seed_for(1, rank), "uniform")
    x_host = torch.from_numpy(x_np).to(tdt).pin_memory()
    w_host = torch.from_numpy(w_np).to(tdt).pin_memory()
    x = x_host.to(dev)
    w = w_host.to(dev)
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=args.math, io_dtype=io, device=local,
                   kernel=args.kernel)
    info = plan.info()
    y = torch.empty(plan.output_shape, dtype=tdt, device=dev)
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    evict = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)

    def flush_l2():
        flush.zero_()   # > L2: evicts x, w, y
        evict.sum()     # > L2, read-only: writes the dirty flush lines back before the step
    stream = torch.cuda.current_stream()
    K, W = args.steps, args.warmup

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # warm-up
    for _ in range(W):
        flush_l2()
        plan.forward(x, w, y)
    barrier()

    # timed region: K steps, each between events on the launching stream (L2 flushed
    # before each, outside the events).  Then a second pass of K steps in which the
    # library records its own events around the dominant kernel (roofline.kernel_ms);
    # kept separate so the nested events do not inflate the step time.
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for a, b in kev:
        a.record(); b.record()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    with sampler:
        barrier()
        for i in range(K):
            flush_l2()
            ev[i][0].record(stream)
            plan.forward(x, w, y)
            ev[i][1].record(stream)
        barrier()
        for i in range(K):
            flush_l2()
            plan.set_timing_events(*kev[i])
            plan.forward(x, w, y)
        barrier()
    plan.set_timing_events(None, None)
    step_ms = [a.elapsed_time(b) for a, b in ev]
    kern_ms = [a.elapsed_time(b) for a, b in kev]
    t_total = torch.tensor([sum(step_ms), sum(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_total, op=dist.ReduceOp.MAX)
    t_step_ms, t_kern_ms = float(t_total[0]) / K, float(t_total[1]) / K
    F = shape.flops()
    value = F * world / (t_step_ms * 1e-3) / 1e12

    # end to end through the C-ABI host entry point (H2D of x,w + forward + D2H of y per step)
    y_host = torch.empty(plan.output_shape, dtype=tdt).pin_memory()
    Ke = min(K, 100)
    for _ in range(3):
        plan.forward_host(x_host, w_host, y_host)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(Ke):
        plan.forward_host(x_host, w_host, y_host)
    e1.record(stream)
    barrier()
    t_e2e = torch.tensor([e0.elapsed_time(e1) / Ke], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_e2e, op=dist.ReduceOp.MAX)
    e2e_value = F * world / (float(t_e2e) * 1e-3) / 1e12

    # cuDNN through torch on the same device tensors (the bar on the same box)
    cudnn = None
    if not args.no_cudnn:
        cudnn = bench_cudnn(torch, x, w, shape, args.math, flush_l2, min(K, 100), world, dist)

    # parity spot-check of the timed launch (sampled image vs the fp64 oracle) is in tests/;
    # here: a cheap sanity check that the output is finite
    if not bool(torch.isfinite(y.float()).all()):
        raise SystemExit("non-finite output")

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    peaks, src = _peaks()
    bound, peak, peak_note = _roofline_peak(args.math, peaks)
    achieved = F / (t_kern_ms * 1e-3) / 1e12
    eb_w = eb
    alg_bytes = shape.bytes(eb, eb_w, eb)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": W,
        "ms_per_step": t_step_ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": args.math, "data": "synthetic",
        "config": {"workload": shape.name, "N": shape.N, "C": shape.C, "K": shape.K, "H": shape.H, "W": shape.W,
                   "R": shape.R, "S": shape.S, "stride": list(shape.stride), "padding": list(shape.padding),
                   "io_dtype": io, "math": args.math, "kernel": info["kernel"],
                   "tile": [info["tile_m"], info["tile_n"], info["stages"]], "per_rank_batch": shape.N,
                   "parallelism": "batch-sharded x%d (weak, no collective)" % world,
                   "l2": "flushed between steps (256 MiB write, then 256 MiB read so no dirty lines remain)", "inputs": "seeded synth 'uniform'"},
        "roofline": {"bound": bound, "achieved": achieved, "peak": peak,
                     "unit": "TFLOP/s", "frac": achieved / peak, "traffic": _traffic("mac_%s_%s" % (info["kernel"], args.math)),
                     "traffic_l2_write": _traffic("mac_%s_%s" % (info["kernel"], args.math), "l2_write"),
                     "traffic_note": "traffic = the launch's dram read + write (ncu); y stays dirty in L2 at the "
                                     "end of the launch, so its write-back shows in traffic_l2_write instead",
                     "algorithmic_bytes": alg_bytes,
                     "kernel": "mac_%s" % info["kernel"], "kernel_ms": t_kern_ms,
                     "kernel_timing": "CUDA events recorded by the library around its launch (own pass of K steps)",
                     "algorithmic": "2*N*K*C*R*S*P*Q = %.4g FLOP per launch" % F,
                     "peak_source": "%s (%s)" % (peak_note, src),
                     "hbm_floor_ms": alg_bytes / (peaks["hbm_gbs"] * 1e9) * 1e3,
                     "step_frac": F / (t_step_ms * 1e-3) / 1e12 / peak},
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(x.numel() * eb + w.numel() * eb),
                "d2h_bytes_per_step": int(y.numel() * eb), "ms_per_step": float(t_e2e),
                "api": "polyconv_forward_host"},
        "gpu_launches": int(info["launches"]) * K,
        "clocks": sampler.summary(),
    }
    if cudnn:
        line["cudnn"] = cudnn
        line["cudnn"]["ratio_ours_over_cudnn"] = value / cudnn["value"]
    if world == 1 and not args.no_gate and args.math == "bf16" and args.workload == "conv3x":
        line["gate"] = bench_gate(torch, pc, dev, flush_l2, peaks, 20, not args.no_cudnn)
    if world == 1 and not args.no_by_math and args.math == "bf16" and args.workload == "conv3x":
        line["by_math"] = bench_by_math(torch, pc, dev, shape, flush_l2, peaks, 20)
    if world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(shape)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0



# ------------------------------------------------------------ gate and by_math --

GATE_LAYERS = [L for L in synth.RESNET50 if L.R == 3 and L.stride == (1, 1)]   # 13 convs, 4 shapes


def _time_fn(torch, fn, flush, reps, warm=3):
    for _ in range(warm):
        flush()
        fn()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        flush()
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    ts = sorted(a.elapsed_time(b) for a, b in evs)
    return ts[len(ts) // 2], sum(ts) / len(ts)


def bench_gate(torch, pc, dev, flush, peaks, reps, with_cudnn):
    """north_star gate: the 13 stride-1 3x3 convs of ResNet-50 at N=256 (BASELINE.json configs[4])
    on one GPU, BF16 in/out and math, L2 flushed before every call.  Per layer: median time,
    effective TFLOP/s, roofline time max(F/peak_bf16, B/HBM) and its fraction; aggregate
    gate_frac = sum(count*roof) / sum(count*t)."""
    import torch.nn.functional as Fn
    recs = []
    roof_sum = t_sum = 0.0
    for li, L in enumerate(GATE_LAYERS):
        g = torch.Generator(device=dev).manual_seed(synth.seed_for(4, li))
        x = (torch.rand((L.N, L.C, L.H, L.W), device=dev, generator=g) * 2 - 1).bfloat16()
        w = ((torch.rand((L.K, L.C, L.R, L.S), device=dev, generator=g) * 2 - 1) / (L.C * L.R * L.S) ** 0.5).bfloat16()
        plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="bf16", io_dtype="bf16", device=dev.index)
        y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device=dev)
        t_med, t_mean = _time_fn(torch, lambda: plan.forward(x, w, y), flush, reps)
        F = L.flops()
        B = L.bytes(2, 2, 2)
        roof_ms = max(F / (peaks["bf16_tflops"] * 1e12), B / (peaks["hbm_gbs"] * 1e9)) * 1e3
        rec = {"layer": L.name, "count": L.count, "shape": [L.N, L.C, L.H, L.W, L.K, L.R, L.S],
               "kernel": plan.info()["kernel"], "t_med_ms": t_med, "t_mean_ms": t_mean,
               "tflops": F / (t_med * 1e-3) / 1e12, "roof_ms": roof_ms, "frac": roof_ms / t_med,
               "bound": "tensor" if F / (peaks["bf16_tflops"] * 1e12) >= B / (peaks["hbm_gbs"] * 1e9) else "hbm"}
        if with_cudnn:
            torch.backends.cudnn.benchmark = True
            best = None
            for layout in ("nchw", "channels_last"):
                xx, ww = (x, w) if layout == "nchw" else (x.contiguous(memory_format=torch.channels_last),
                                                           w.contiguous(memory_format=torch.channels_last))
                tc, _ = _time_fn(torch, lambda: Fn.conv2d(xx, ww, stride=L.stride, padding=L.padding), flush,
                                 max(5, reps // 2))
                v = F / (tc * 1e-3) / 1e12
                rec["cudnn_%s_tflops" % layout] = v
                if best is None or v > best[0]:
                    best = (v, layout)
            rec["cudnn_best_tflops"], rec["cudnn_best_layout"] = best
        recs.append(rec)
        roof_sum += L.count * roof_ms
        t_sum += L.count * t_med
        del plan, x, w, y
    return {"layers": recs, "gate_frac": roof_sum / t_sum, "convs": sum(L.count for L in GATE_LAYERS),
            "target": 0.60, "peak_tflops": peaks["bf16_tflops"], "hbm_gbs": peaks["hbm_gbs"],
            "note": "ResNet-50 N=256 stride-1 3x3 convs on one GPU, BF16, L2 flushed, median of %d" % reps}


def bench_by_math(torch, pc, dev, shape, flush, peaks, reps):
    """conv3x (BASELINE configs[1]) in the other two maths (fp32 I/O): TF32 tensor cores and the
    FP32 FFMA path (the paper's inferred precision), each against its own roofline."""
    out = {}
    x_np, w_np = synth.make_inputs(shape, synth.seed_for(1), "uniform")
    x = torch.from_numpy(x_np).to(dev)
    w = torch.from_numpy(w_np).to(dev)
    for math in ("tf32", "fp32"):
        plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype="f32", device=dev.index)
        y = torch.empty(plan.output_shape, dtype=torch.float32, device=dev)
        t_med, t_mean = _time_fn(torch, lambda: plan.forward(x, w, y), flush, reps)
        bound, peak, note = _roofline_peak(math, peaks)
        F = shape.flops()
        B = shape.bytes(4, 4, 4)
        roof_ms = max(F / (peak * 1e12), B / (peaks["hbm_gbs"] * 1e9)) * 1e3
        out[math] = {"value": F / (t_mean * 1e-3) / 1e12, "unit": UNIT, "t_mean_ms": t_mean, "t_med_ms": t_med,
                     "kernel": plan.info()["kernel"], "bound": bound, "peak": peak, "peak_source": note,
                     "frac": roof_ms / t_mean, "io_dtype": "f32"}
        del plan, y
    return out

def bench_cudnn(torch, x, w, shape, math, flush, K, world, dist):
    import torch.nn.functional as Fn
    torch.backends.cudnn.benchmark = True
    torch.backends.cudnn.allow_tf32 = math == "tf32"
    best = None
    by_layout = {}
    for layout in ("nchw", "channels_last"):
        xx, ww = (x, w) if layout == "nchw" else (x.contiguous(memory_format=torch.channels_last),
                                                   w.contiguous(memory_format=torch.channels_last))
        for _ in range(5):
            Fn.conv2d(xx, ww, stride=shape.stride, padding=shape.padding)
        torch.cuda.synchronize()
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        for a, b in evs:
            flush()
            a.record()
            Fn.conv2d(xx, ww, stride=shape.stride, padding=shape.padding)
            b.record()
        torch.cuda.synchronize()
        t = torch.tensor([sum(a.elapsed_time(b) for a, b in evs) / K], dtype=torch.float64, device=x.device)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        v = shape.flops() * world / (float(t) * 1e-3) / 1e12
        by_layout[layout] = {"value": v, "ms_per_step": float(t)}
        if best is None or v > best["value"]:
            best = {"value": v, "unit": UNIT, "ms_per_step": float(t), "layout": layout,
                    "library": "cuDNN %s via torch.nn.functional.conv2d (benchmark=True)" %
                    torch.backends.cudnn.version()}
    # nchw = the same NCHW tensors this library takes; channels_last = cuDNN's preferred
    # layout (input converted outside the timed region)
    best["by_layout"] = by_layout
    return best


if __name__ == "__main__":
    sys.exit(main())
