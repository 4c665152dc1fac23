#!/usr/bin/env python
"""bench.py -- KAMI batched small-GEMM throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl kami|reference]
                    [--workload f16-64 | f16-32 | f16-128 | f16-16 | f64-16 | f64-32 | f64-64 |
                                lr-8 | lr-16 | lr-32 | bf16-<m>x<n>x<k>] [--algo auto|1d|2d|3d|nonca]
    torchrun --nproc-per-node N bench.py --gpus N ...

A "step" is one pass of the whole hot path over one batch: one
kami_gemm_strided_batched call (plan -> TMA/LDG loads -> CA exchange -> MMA ->
store) over the workload's batch of resident device inputs.  Default
workload = BASELINE.json configs[1] at its headline order: FP16 in / FP32
accumulate, m=n=k=64, batch 65 536 per GPU (weak scaling: every rank owns its
own 65 536 entries; entries are generated on the device by the shared
counter-based generator keyed by global entry index).

Prints ONE JSON line (rank 0).  value = whole-job TFLOP/s (2mnk per entry,
padding not counted) over the max-over-ranks device time of K steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "batched small-GEMM TFLOP/s and % roofline (fp16/fp64) at 1/2/4/8 B200"

WORKLOADS = {
    # name: (dtype, m, n, k, batch per GPU, BASELINE config index)
    "f16-16": ("f16", 16, 16, 16, 1024, 0),
    "f16-32": ("f16", 32, 32, 32, 65536, 1),
    "f16-64": ("f16", 64, 64, 64, 65536, 1),
    "f16-128": ("f16", 128, 128, 128, 65536, 1),
    "f64-16": ("f64", 16, 16, 16, 32768, 2),
    "f64-32": ("f64", 32, 32, 32, 32768, 2),
    "f64-64": ("f64", 64, 64, 64, 32768, 2),
    "lr-8": ("f16", 256, 256, 8, 16384, 3),
    "lr-16": ("f16", 256, 256, 16, 16384, 3),
    "lr-32": ("f16", 256, 256, 32, 16384, 3),
    # SURVEY f4 variants (not BASELINE configs; same shape as configs[1] 64^3)
    "tf32-64": ("tf32", 64, 64, 64, 65536, 1),
    "e4m3-64": ("e4m3", 64, 64, 64, 65536, 1),
    "e5m2-64": ("e5m2", 64, 64, 64, 65536, 1),
    "f16upd-64": ("f16", 64, 64, 64, 65536, 1),   # C = A B + C (beta = 1: C read and written)
}
ES_IN = {"f64": 8, "tf32": 4, "e4m3": 1, "e5m2": 1}
ES_OUT = {"f64": 8, "tf32": 4}


def op_bytes(dtype, m, n, k, update=False):
    """Algorithmic bytes of one entry: A, B read once, C written once (and
    read once more when beta != 0)."""
    return (m * k + k * n) * ES_IN.get(dtype, 2) + m * n * ES_OUT.get(dtype, 2) * (2 if update else 1)


def parse_workload(name):
    if name in WORKLOADS:
        return WORKLOADS[name]
    dt, _, rest = name.partition("-")
    if dt in ("bf16", "f16", "f64") and "x" in rest:  # <dtype>-<m>x<n>x<k>[:batch]
        spec, _, b = rest.partition(":")
        m, n, k = (int(x) for x in spec.split("x"))
        default = {"bf16": (125000, 4), "f16": (65536, 1), "f64": (32768, 2)}[dt]
        return (dt, m, n, k, int(b) if b else default[0], default[1])
    raise SystemExit(f"unknown workload {name}")


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6650.0), d.get("bf16_tflops", 1590.0), "measured (MEASURED_PEAKS.json)"
    return 6650.0, 1590.0, "fallback (B200_PROFILING.md)"


_FP64_PEAK = {}


def fp64_peak_tflops():
    """FP64 DMMA roofline denominator, MEASURED on this device by the library's
    probe (kami_probe_dmma_peak: an mma.sync.m8n8k4.f64 loop on every SM for
    >= 300 ms; MEASURED_PEAKS.json has no FP64 figure).  The sustained rate
    (second half of the run, clock under the power cap) is the denominator for
    kernels timed inside a long step; falls back to the 37 TF/s nominal figure
    (148 SMs x 1965 MHz x the DMMA issue rate) if the probe cannot run."""
    if not _FP64_PEAK:
        try:
            import paper_conf_sc_wangdltsl25_b200 as kami

            burst, sus = kami.probe_dmma_peak(300.0)
            _FP64_PEAK.update(value=sus, burst=burst, source="measured (kami_probe_dmma_peak, sustained)")
        except Exception as e:  # pragma: no cover
            _FP64_PEAK.update(value=37.0, burst=None, source=f"nominal 37 TF/s (probe failed: {e})")
    return _FP64_PEAK["value"]


class ClockSampler:
    """nvidia-smi clocks/throttle sampler run DURING the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,clocks.mem,"
         "temperature.gpu,temperature.memory")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for nm, v in zip(names, r[5:9]):
                if v.strip().lower() == "active":
                    reasons.add(nm)
        def med(i):
            v = [float(r[i]) for r in self.rows if len(r) > i and r[i].replace(".", "").isdigit()]
            return statistics.median(v) if v else None
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows), "mem_mhz": med(9), "power_w": med(3),
                "gpu_temp_c": med(10), "mem_temp_c": med(11)}


def host_cpu_info():
    """CPU model, logical CPUs (nproc) and the affinity mask size (the threads
    the oracle may actually use) -- BASELINE.md 4 / SURVEY.md 8(d)."""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    try:
        aff = len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        aff = os.cpu_count()
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity": aff}


def cpu_baseline(dtype, m, n, k, target_s=12.0, max_entries=None):
    """Time the oracle (as it stands) on this host's cores on a bounded sample,
    plus a 1-thread rate on a smaller sample (per-core baseline)."""
    import kami_inputs as ki
    import oracle

    cores = oracle.default_threads()
    per_entry_mac = m * n * k
    # calibrate on a small sample, then size the sample to ~target_s
    probe = max(cores, int(2e7 // per_entry_mac) or 1)
    A, B = ki.operands(m, n, k, probe, dtype, "unif", seed=0)
    a, b = ki.as_bits(A), ki.as_bits(B)
    t0 = time.perf_counter()
    oracle.gemm(m, n, k, probe, dtype, "row", a, b, nthreads=cores)
    dt = time.perf_counter() - t0
    n_entries = max(probe, int(probe * target_s / max(dt, 1e-6)))
    if max_entries:
        n_entries = min(n_entries, max_entries)
    A, B = ki.operands(m, n, k, n_entries, dtype, "unif", seed=0)
    a, b = ki.as_bits(A), ki.as_bits(B)
    t0 = time.perf_counter()
    oracle.gemm(m, n, k, n_entries, dtype, "row", a, b, nthreads=cores)
    dt = time.perf_counter() - t0
    tflops = 2.0 * per_entry_mac * n_entries / dt / 1e12
    # one thread on ~1/8 of the time budget
    n1 = max(1, min(n_entries, int(n_entries / cores * (target_s / 8) / max(dt, 1e-6))))
    t0 = time.perf_counter()
    oracle.gemm(m, n, k, n1, dtype, "row", a[: n1 * m * k], b[: n1 * k * n], nthreads=1)
    dt1 = time.perf_counter() - t0
    out = {"value": tflops, "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
           "sample": f"first {n_entries} entries of the workload (seed 0), FP64 triple loop, {dt:.1f} s",
           "seconds": dt, "entries": n_entries,
           "one_thread": {"value": 2.0 * per_entry_mac * n1 / dt1 / 1e12, "unit": "TFLOP/s", "entries": n1,
                          "seconds": dt1}}
    out.update(host_cpu_info())
    return out


PAPER_CONTEXT = {
    "note": "KAMI (SC'25) prints no absolute batched TFLOP/s (Fig. 12 is an image); other hardware, not a target",
    "batched_fp64_gh200": "avg 31.60x vs MAGMA 2.9, 340.37x vs cuBLAS 12.8 at batch 1000 (orders 16-128; P:L525)",
    "block_level_fp64_gh200": "cuBLASDx 64x64 31 TFLOP/s = 46% of the 67 TF peak (P:L90, P:L95)",
    "block_level_fp16_rtx5090": "KAMI-1D/2D/3D 64x64 469.80/470.57/449.07 TFLOP/s (P:L484)",
    "hardware": "NVIDIA GH200 (FP16 990 TF, FP64 67 TF), RTX 5090 (FP16 462 TF), AMD 7900 XTX, Intel Max 1100 "
                "(PAPER.md L49, Table 3); the non-NVIDIA results are reported as speedups only",
}


def dist_init():
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and os.environ.get("KAMI_BENCH_SHARED_GPU") == "1":
        # test mode only (never the measured run): N ranks on one GPU, so the
        # multi-rank path (shards, barriers, max over ranks, stats gather) can
        # be exercised on a 1-GPU box; NCCL refuses two ranks on one device, so
        # the stats travel over gloo
        torch.cuda.set_device(local % torch.cuda.device_count())
        dist.init_process_group("gloo")
    elif world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    return world, rank, local


def run_reference(args):
    """--impl reference: the oracle timed on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    dtype, m, n, k, batch, cfg = parse_workload(args.workload)
    import kami_inputs as ki
    import oracle

    cores = oracle.default_threads()
    # each step = a bounded sample of the workload sized so the run takes ~1-2 min
    per_entry = 2.0 * m * n * k
    probe = max(cores, int(2e7 // (m * n * k)) or 1)
    A, B = ki.operands(m, n, k, probe, dtype, "unif")
    t0 = time.perf_counter()
    oracle.gemm(m, n, k, probe, dtype, "row", ki.as_bits(A), ki.as_bits(B), nthreads=cores)
    rate = probe / max(time.perf_counter() - t0, 1e-6)
    steps_total = args.steps + args.warmup
    sample = max(cores, min(batch, int(rate * 90.0 / steps_total)))
    A, B = ki.operands(m, n, k, sample, dtype, "unif")
    a, b = ki.as_bits(A), ki.as_bits(B)
    for _ in range(args.warmup):
        oracle.gemm(m, n, k, sample, dtype, "row", a, b, nthreads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.gemm(m, n, k, sample, dtype, "row", a, b, nthreads=cores)
    dt = (time.perf_counter() - t0) / args.steps
    value = per_entry * sample / dt / 1e12
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": dtype, "data": "synthetic",
        "config": dict(workload_config(args, dtype, m, n, k, batch, cfg), timing="host wall clock"),
        "cpu_baseline": dict({"value": value, "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
                              "sample": f"{sample} entries of the workload per step (of {batch}), FP64 triple loop"},
                             **host_cpu_info()),
        "e2e": {"value": value, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(args, dtype, m, n, k, batch, cfg):
    return {"workload": f"{dtype} strided-batched GEMM m={m} n={n} k={k} batch={batch}/GPU row-major "
                        f"(BASELINE.json configs[{cfg}])",
            "m": m, "n": n, "k": k, "batch_per_gpu": batch, "global_batch": getattr(args, "global_batch", batch),
            "scaling": getattr(args, "scaling", "weak"),
            "layout": "row", "algo": args.algo, "p": args.p, "inputs": "unif [-1,1) RNE to dtype, counter-based SplitMix64",
            "l2": "inputs larger than L2 (126 MB)" if batch * op_bytes(dtype, m, n, k) >= 126e6
                  else f"inputs rotated over {int(-(-3 * 126e6 // (batch * op_bytes(dtype, m, n, k))))} distinct "
                       "sets (> 3x the 126 MB L2); L2 evicted by a 252 MB write before the timed region",
            "timing": {"graph": "K steps captured in one CUDA graph, replayed between two CUDA events on the "
                                "launch stream",
                       "b2b": "K steps launched back to back between two CUDA events on the launch stream",
                       "events": "one CUDA event pair per step on the launch stream, summed"}[args.timing],
            "parallelism": f"batch-sharded dp{args.gpus}"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="kami", choices=["kami", "reference"])
    ap.add_argument("--workload", default="f16-64")
    ap.add_argument("--algo", default="auto")
    ap.add_argument("--p", type=int, default=0, help="warps per entry (0 = planner default)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: the workload batch per GPU; strong: the workload batch split over the GPUs")
    ap.add_argument("--timing", default="graph", choices=["graph", "b2b", "events"],
                    help="graph: K steps in one CUDA graph between two events; b2b: K launches back to back "
                         "between two events; events: one event pair per launch, summed")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import kami_inputs as ki
    import paper_conf_sc_wangdltsl25_b200 as kami

    from paper_conf_sc_wangdltsl25_b200 import dist as kdist

    world, rank, local = dist_init()
    dtype, m, n, k, wl_batch, cfg = parse_workload(args.workload)
    # this rank's contiguous slice of the global batch (dist.py):
    # weak scaling = the workload batch per GPU, strong = the workload batch in total
    if args.scaling == "strong":
        lo, hi = kdist.shard_range(wl_batch, rank, world)
        global_batch = wl_batch
    else:
        lo, hi = kdist.weak_range(wl_batch, rank)
        global_batch = wl_batch * world
    batch = hi - lo
    args.global_batch = global_batch
    update = "upd" in args.workload
    esi, eso = ES_IN.get(dtype, 2), ES_OUT.get(dtype, 2)
    alg_bytes = batch * op_bytes(dtype, m, n, k, update)
    flops = 2.0 * m * n * k * batch
    # L2-resident workloads (configs[0]: 1.5 MB) rotate over R distinct input /
    # output sets whose total exceeds 3x the 126 MB L2, so every timed step
    # reads cold inputs without an L2 flush inside the timed region
    R = 1 if alg_bytes >= 126e6 else int(-(-3 * 126e6 // alg_bytes))
    sets = []
    for r_ in range(R):
        entry0 = lo + r_ * global_batch  # set 0 = this rank's entries of the global batch
        A, B = ki.operands(m, n, k, batch, dtype, "unif", seed=0, entry0=entry0, device="cuda")
        C = torch.zeros(batch * m * n, dtype=ki.TORCH_DTYPES[ki.OUT_DTYPE[dtype]], device="cuda")
        sets.append((A, B, C))
    A, B, C = sets[0]
    stream = torch.cuda.current_stream()

    def step(i=0):
        A_, B_, C_ = sets[i % R]
        st = torch.cuda.current_stream()  # the capture stream while a graph is being recorded
        if update:  # C <- A B + C
            kami.gemm_strided_batched_axpby(m, n, k, batch, dtype, "row", 1.0, A_, B_, 1.0, C_, stream=st)
        else:
            kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A_, B_, C_, algo=args.algo, p=args.p,
                                      stream=st)

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    kernel = kami.last_kernel()

    # clocks sampled during a ~1.5 s sustained burst plus the timed region
    sampler = ClockSampler(torch.cuda.current_device())
    sampler.start()
    t_end = time.time() + 1.5
    while time.time() < t_end:
        for i in range(20):
            step(i)
        torch.cuda.synchronize()

    # The K steps are captured once into a CUDA graph (the launch-bound small
    # configs would otherwise time the host's per-call cost, ~10 us, instead of
    # the kernels) and replayed between one pair of events on the launch
    # stream; the per-step average is the kernel's launch duration, gaps
    # between launches included.  --timing b2b / events for comparison.
    graph = None
    if args.timing == "graph":
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            for i in range(args.steps):
                step(i)
        graph.replay()  # untimed
        torch.cuda.synchronize()
    if R > 1:
        # the untimed replay just touched the same input sets the timed replay
        # reads first: evict L2 (a 2 x 126 MB write) outside the timed region so
        # every timed step reads cold inputs (the R sets exceed 3x L2, so sets
        # reused later in the K steps are cold as well)
        flush = torch.empty(2 * 126 * 1024 * 1024, dtype=torch.uint8, device="cuda")
        flush.fill_(1)
        torch.cuda.synchronize()
        del flush
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if args.timing == "events":
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(args.steps)]
        for i, (e0, e1) in enumerate(evs):
            e0.record(stream)
            step(i)
            e1.record(stream)
    else:
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        if graph is not None:
            graph.replay()
        else:
            for i in range(args.steps):
                step(i)
        ev1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    sampler.stop()
    if args.timing == "events":
        t_ms = sum(a.elapsed_time(b) for a, b in evs)
    else:
        t_ms = ev0.elapsed_time(ev1)  # device time of the K timed steps

    # world-size-invariant checksum of this rank's outputs (set 0 = its entries
    # [lo, hi) of the global batch; parity itself is checked in tests/), then
    # the only collective: an all_gather of the tiny per-rank record (dist.py)
    csum = kdist.position_checksum(C, lo, batch, m * n)
    coll_dev = "cpu" if world > 1 and dist.get_backend() == "gloo" else "cuda"
    recs = kdist.gather_records(kdist.RankRecord(time_ms=t_ms, checksum=float(csum), entries=float(batch)),
                                device=coll_dev)
    agg = kdist.aggregate(recs)
    t_max_ms = agg["time_ms"]
    total_entries = agg["entries"]

    # end-to-end: the C-ABI host entry point, host<->device copies inside the timed region
    e2e = None
    if not args.no_e2e and not update:
        hA = A.cpu().pin_memory()
        hB = B.cpu().pin_memory()
        hC = torch.empty(C.numel(), dtype=C.dtype).pin_memory()
        kami.gemm_strided_batched_host(m, n, k, batch, dtype, "row", hA, hB, hC)  # warm (workspace)
        if world > 1:
            dist.barrier()
        e_steps = 3
        t0 = time.perf_counter()
        for _ in range(e_steps):
            kami.gemm_strided_batched_host(m, n, k, batch, dtype, "row", hA, hB, hC)
        e_dt = (time.perf_counter() - t0) / e_steps
        et = torch.tensor([e_dt], dtype=torch.float64, device=coll_dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e = {"value": flops * world / float(et.item()) / 1e12, "unit": "TFLOP/s",
               "h2d_bytes_per_step": batch * (m * k + k * n) * esi, "d2h_bytes_per_step": batch * m * n * eso,
               "path": "kami_gemm_strided_batched_host (pinned host buffers, chunked H2D/kernel/D2H pipeline)"}
        kami.release_workspace()

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    hbm, bf16pk, peak_src = load_peaks()
    value = flops * total_entries / batch * args.steps / (t_max_ms * 1e-3) / 1e12
    avg_launch_s = (t_ms / args.steps) * 1e-3
    achieved_gbs = alg_bytes / avg_launch_s / 1e9
    tensor_peak = fp64_peak_tflops() if dtype == "f64" else {"tf32": 1125.0, "e4m3": 4500.0, "e5m2": 4500.0}.get(
        dtype, 2250.0)
    roof_tf = min(hbm * 1e9 * flops / alg_bytes, tensor_peak * 1e12) / 1e12
    bound = "hbm"
    if dtype == "f64" and fp64_peak_tflops() * 1e12 < hbm * 1e9 * flops / alg_bytes:
        bound = "tensor"
    if bound == "hbm":
        roofline = {"bound": "hbm", "achieved": achieved_gbs, "peak": hbm, "unit": "GB/s",
                    "frac": achieved_gbs / hbm, "peak_source": peak_src}
    else:
        ach = flops / avg_launch_s / 1e12
        roofline = {"bound": "tensor", "achieved": ach, "peak": fp64_peak_tflops(), "unit": "TFLOP/s",
                    "frac": ach / fp64_peak_tflops(), "peak_source": _FP64_PEAK["source"],
                    "peak_burst": _FP64_PEAK["burst"]}
    roofline["traffic"] = traffic_from_profiles(args.workload)
    roofline["kernel"] = kernel
    roofline["roofline_tflops_per_gpu"] = roof_tf
    roofline["frac_of_roofline_tflops"] = (value / world) / roof_tf
    line = {
        "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_max_ms / args.steps, "higher_is_better": True,
        "scaling": args.scaling,
        "vs_baseline": None, "dtype": dtype, "data": "synthetic",
        "config": workload_config(args, dtype, m, n, k, batch, cfg),
        "roofline": roofline,
        "gpu_launches": args.steps,
        "clocks": sampler.summary(),
        # position-weighted checksum of every output bit pattern, exactly additive
        # over shards: identical for any world size / scaling mode on the same
        # global entries (dist.position_checksum)
        "checksum": agg["position_checksum"],
    }
    if world > 1:  # per-rank device times (the job time is their max)
        line["ranks"] = {"time_ms": [r.time_ms for r in recs], "spread": agg["spread"],
                         "entries": [int(r.entries) for r in recs], "checksums": [int(r.checksum) for r in recs]}
    if e2e:
        line["e2e"] = e2e
    # the paper's own numbers, other hardware: context only (vs_baseline stays null)
    line["paper_context"] = PAPER_CONTEXT
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(dtype, m, n, k)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def traffic_from_profiles(workload):
    """dram bytes (read + write) per launch of the dominant kernel from the
    committed ncu --set full summary (profiles/*/ncu_summary.json), or None."""
    pdir = os.path.join(ROOT, "profiles")
    best = None
    if os.path.isdir(pdir):
        for d in sorted(os.listdir(pdir)):
            f = os.path.join(pdir, d, "ncu_summary.json")
            if os.path.exists(f):
                try:
                    s = json.load(open(f))
                    if workload in s.get("traffic_bytes_per_launch", {}):
                        best = s["traffic_bytes_per_launch"][workload]
                except Exception:
                    pass
    return best


if __name__ == "__main__":
    main()
