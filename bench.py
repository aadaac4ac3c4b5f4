#!/usr/bin/env python
"""GLP label-propagation benchmark (BASELINE.json metric: LP edges/sec per
iteration, GTEPS, and time-to-converge).

One *step* = one complete ``glp_run`` of the north_star hot path on a
device-resident graph: PickLabel, then synchronous MFL iterations (gather ->
count -> arg-max -> update, active-vertex frontier, exact stop rule) until a
fixed point, a two-cycle or the paper's 20 iterations [P:270].

  value  = GTEPS = arcs actually scanned over the run / device time of the run
           (GTEPS_t = sum of the degrees of the vertices scanned
           at t, counting only the arcs whose labels were gathered -- a row
           that stops on a strict majority is credited with the arcs it
           read); the paper's "average elapsed time for one iteration"
           [P:355] as a rate.  nnz x iterations / time is reported beside it
           as `nnz_x_iterations_gteps` (it credits arcs the frontier skipped)
  e2e    = the same metric through the public C ABI with HOST buffers:
           glp_graph_create(host CSR) + glp_run + glp_labels_get(host) per step

Default workload (N=1): RMAT scale-24, edge factor 16, classic LP
(BASELINE.json configs[2], the north_star's roofline config).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload rmat24]
  python bench.py --impl reference ...   # the CPU oracle arm (bounded sample)
Under torchrun (N>1) the graph is 1-D vertex-partitioned across ranks with the
NCCL label all-gather (strong scaling); rank 0 prints the JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "LP edges/sec per iteration (GTEPS) and time-to-converge"
UNIT = "GTEPS"

WORKLOADS = {
    # name: (generator spec, variant, max_iters, gamma)
    "rmat24": (dict(kind="rmat", scale=24, edge_factor=16, seed=1), "classic", 20, 0.0),
    "sbm1m": (dict(kind="sbm", n=1_000_000, k=1000, m=20_000_000, mu=0.1, seed=42), "classic", 30, 0.0),
    "taobao100m": (dict(kind="taobao", users=80_000_000, items=20_000_000, pairs=1_000_000_000, seed=7),
                   "seeded", 20, 0.0),
    "rmat24_llp": (dict(kind="rmat", scale=24, edge_factor=16, seed=1), "llp", 20, 1.0),
    "rmat28_llp": (dict(kind="rmat", scale=28, edge_factor=16, seed=1, buckets=16), "llp", 20, 1.0),
    "karate": (dict(kind="karate"), "classic", 20, 0.0),
    # §8(f)4 hybrid mode: the same RMAT-24 run with the arc array in pinned host
    # memory, streamed over the host link every iteration
    "rmat24_hostarcs": (dict(kind="rmat", scale=24, edge_factor=16, seed=1), "classic", 20, 0.0),
}
HOST_ARCS = {"rmat24_hostarcs"}
# §8(f)3 weighted LP: RMAT-24 with symmetric integer arc weights in [1, 8]
WORKLOADS["rmat24_weighted"] = (dict(kind="rmat", scale=24, edge_factor=16, seed=1), "classic", 20, 0.0)
WEIGHTED = {"rmat24_weighted"}
# §8(f)3 SLP: 5 candidate labels, 20 iterations [P:270]
WORKLOADS["rmat24_slp"] = (dict(kind="rmat", scale=24, edge_factor=16, seed=1), "slp", 20, 0.0)


def host_link_gbs(dev) -> float:
    """Measured pinned host -> device copy bandwidth (GB/s), the hybrid
    mode's roofline denominator."""
    import torch
    h = torch.empty(1 << 28, dtype=torch.int32).pin_memory()
    d = torch.empty(1 << 28, dtype=torch.int32, device=dev)
    best = 0.0
    for _ in range(4):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        d.copy_(h, non_blocking=True)
        e1.record()
        e1.synchronize()
        best = max(best, h.numel() * 4 / (e0.elapsed_time(e1) / 1e3) / 1e9)
    return best


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy bandwidth)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled every 200 ms while running."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.path = None

    def __enter__(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except (OSError, FileNotFoundError):
            self.proc = None
        return self

    def __exit__(self, *exc):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if self.proc is None or not self.path or not os.path.exists(self.path):
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                smax = float(parts[2])
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        os.unlink(self.path)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


def make_graph(spec, device):
    from glp_inputs import graphs
    csr, seeds = graphs.make(spec["kind"], device=device, **{k: v for k, v in spec.items() if k != "kind"})
    return csr, seeds


def workload_weights(name, csr):
    if name not in WEIGHTED:
        return None
    from glp_inputs import graphs
    return graphs.edge_weights(csr, seed=5, hi=8)


def cpu_reference(csr_cpu, variant, seeds, gamma, iters_per_sample, reps, warmup=0, weights=None):
    """Time the CPU oracle (as it stands) on the host cores: `reps` samples of
    `iters_per_sample` LP iterations from PickLabel."""
    import oracle
    threads = os.cpu_count() or 1
    vid = {"classic": oracle.CLASSIC, "seeded": oracle.SEEDED, "llp": oracle.LLP, "slp": None}[variant]
    times = []
    for r in range(warmup + reps):
        t0 = time.perf_counter()
        sd = None if seeds is None else seeds.cpu().numpy()
        if variant == "slp":
            oracle.run_slp(csr_cpu, K=5, r=0.0, max_iters=iters_per_sample, threads=threads)

            class _R:
                iterations = iters_per_sample
            res = _R()
        elif weights is not None:
            res = oracle.run_weighted(csr_cpu, weights.cpu().numpy().astype("uint32"), vid, iters_per_sample,
                                      seeds=sd, threads=threads)
        else:
            res = oracle.run(csr_cpu, vid, iters_per_sample, seeds=sd, gamma=gamma, threads=threads)
        dt = time.perf_counter() - t0
        if r >= warmup:
            times.append((dt, res.iterations))
    tot_t = sum(t for t, _ in times)
    tot_it = sum(i for _, i in times)
    value = csr_cpu.nnz * tot_it / tot_t / 1e9 if tot_t > 0 else 0.0
    return value, threads, tot_t / max(len(times), 1), tot_it


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def cpu_sequential(csr_cpu, variant, seeds, gamma, arc_budget=150_000_000):
    """The oracle's per-vertex rule on ONE core (oracle.step, threads=1) for
    iteration 1 from PickLabel, on the first rows holding ~arc_budget arcs
    (a bounded sample; arcs/s of the sequential program)."""
    import numpy as np

    import oracle
    vid = {"classic": oracle.CLASSIC, "seeded": oracle.SEEDED, "llp": oracle.LLP}[variant]
    n = csr_cpu.n
    off, _ = csr_cpu.numpy()
    v_end = int(np.searchsorted(off, min(arc_budget, int(off[-1])), side="left"))
    v_end = max(1, min(n, v_end))
    sd = None if seeds is None else seeds.cpu().numpy()
    L0 = oracle.init_labels(n, vid, sd)
    V = np.ones(n, dtype=np.int32) if vid == oracle.LLP else None
    is_seed = None
    if vid == oracle.SEEDED:
        is_seed = np.zeros(n, dtype=np.uint8)
        if sd is not None and len(sd):
            is_seed[sd] = 1
    t0 = time.perf_counter()
    oracle.step(csr_cpu, vid, L0, 0, v_end, V=V, is_seed=is_seed, gamma=gamma, threads=1)
    dt = time.perf_counter() - t0
    arcs = int(off[v_end])
    return {"value": round(arcs / dt / 1e9, 5), "unit": UNIT, "cores": 1, "arcs": arcs, "seconds": round(dt, 2),
            "sample": f"iteration 1 from PickLabel on rows [0, {v_end}) ({arcs} arcs), oracle.step, 1 thread"}


def flush_l2(buf):
    buf.fill_(1)  # 256 MB write > 126 MB L2


def bench_gpu(args):
    # the e2e leg re-creates the graph every step: let the library's memory
    # pool keep a whole graph mapped between creates (TaoBao: ~25 GB)
    os.environ.setdefault("GLP_POOL_KEEP_GB", "64")
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_yelhls21_b200 as glp

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    spec, variant, max_iters, gamma = WORKLOADS[args.workload]
    if args.max_iters is not None:
        max_iters = args.max_iters
    dev = torch.device("cuda", local)
    t_gen = time.perf_counter()
    csr, seeds = make_graph(spec, dev)
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t_gen
    n, nnz = csr.n, csr.nnz
    stream = torch.cuda.current_stream()
    wts = workload_weights(args.workload, csr)

    # torch's cache of the generator's temporaries (~139 GB after TaoBao) is
    # released, so the library's memory pool can keep a whole graph mapped
    torch.cuda.empty_cache()
    # ---- e2e through the public C ABI with host buffers ----
    # Measured before the device-timed region: after the nvidia-smi clock
    # sampler has run, host-buffer creates on the box turned erratic (SBM
    # 8 ms -> 20-150 ms, tools/e2e_var.py smi), unrelated to the library.
    e2e = None
    if rank == 0 and world == 1 and not args.no_e2e:
        off_h = csr.row_offsets.cpu().pin_memory()
        col_h = csr.col_idx.cpu().pin_memory()
        seeds_h = None if seeds is None else seeds.cpu()
        out_h = torch.empty(n, dtype=torch.int32).pin_memory()
        e2e_ms, e2e_arcs, phases = [], 0, []
        e2e_warm = 2  # the first creates grow the stream-ordered pool
        for r in range(e2e_warm + min(args.steps, 3)):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            g2 = glp.Graph(n=n, row_offsets=off_h, col_idx=col_h, symmetric=csr.symmetric, stream=stream,
                           host_arcs=args.workload in HOST_ARCS, weights=None if wts is None else wts.cpu())
            t1 = time.perf_counter()
            ri = g2.run(variant, max_iters, seeds_h, gamma=gamma)
            t2 = time.perf_counter()
            glp.glp_labels_get(g2.handle, out_h)
            t3 = time.perf_counter()
            dt = (t3 - t0) * 1e3
            g2.close()
            if r >= e2e_warm:
                e2e_ms.append(dt)
                e2e_arcs += ri.arcs_processed
                phases.append(((t1 - t0) * 1e3, (t2 - t1) * 1e3, (t3 - t2) * 1e3))
        e2e = {"value": round(e2e_arcs / (sum(e2e_ms) / 1e3) / 1e9, 3), "unit": UNIT,
               "h2d_bytes_per_step": int((n + 1) * 8 + nnz * 4 + (0 if seeds is None else 4 * seeds.numel())
                                         + (0 if wts is None else 4 * nnz)),
               "d2h_bytes_per_step": int(4 * n), "ms_per_step": round(statistics.mean(e2e_ms), 3),
               "includes": "graph create (H2D copy, relayout) + run + labels D2H",
               "phase_ms": {k: round(statistics.mean(p[i] for p in phases), 3)
                            for i, k in enumerate(("create", "run", "labels_get"))},
               "step_ms": [round(x, 3) for x in e2e_ms], "warmup": e2e_warm}
        del off_h, col_h, out_h

    # ---- partition (1-D vertex ranges; equal vertex counts) ----
    if world > 1:
        from paper_conf_sigmod_yelhls21_b200 import dist as gdist
        g = gdist.distributed_graph(csr, stream=stream)
    else:
        if args.workload in HOST_ARCS:
            g = glp.Graph(csr.to("cpu"), device=local, stream=stream, host_arcs=True)
        else:
            g = glp.Graph(csr, device=local, stream=stream, weights=wts)
    info = g.info()
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)

    def one_run(profile=False):
        return g.run(variant, max_iters, seeds, gamma=gamma, profile=profile)

    for _ in range(max(args.warmup, 0)):
        one_run()
    # ---- per-kernel durations (roofline): profiled steps, in which the library
    # serialises the class kernels of an iteration so that each launch's CUDA
    # events bracket that kernel alone (in the timed region below they run
    # concurrently on side streams and per-launch events would include queueing)
    kstats, prof_ms = {}, []
    kprof_steps = max(1, min(args.steps, 5))
    for _ in range(kprof_steps):
        flush_l2(flush)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        one_run(profile=True)
        e1.record(stream)
        e1.synchronize()
        prof_ms.append(e0.elapsed_time(e1))
        for k in g.kernel_stats():
            s = kstats.setdefault(k["name"], dict(ms=0.0, bytes=0.0, arcs=0.0, launches=0))
            s["ms"] += k["ms"]
            s["bytes"] += k["bytes"]
            s["arcs"] += k["arcs"]
            s["launches"] += k["launches"]
    # ---- timed region: K steps, each bracketed by CUDA events on the run stream ----
    step_ms, infos = [], []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            flush_l2(flush)
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            ri = one_run(profile=False)
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
            infos.append(ri)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    iters = infos[-1].iterations
    arcs_total = nnz if world == 1 else None
    if world > 1:
        t = torch.tensor([csr.nnz], dtype=torch.int64, device=dev)
        arcs_total = csr.nnz  # every rank generated the full graph
    ms_per_step = total_ms / args.steps
    # (with several ranks the library all-reduces its per-iteration counters,
    # so every rank's arcs_processed is already the whole job's)
    scanned = sum(i.arcs_processed for i in infos)
    value = scanned / (total_ms / 1e3) / 1e9
    nnz_iters = arcs_total * sum(i.iterations for i in infos) / (total_ms / 1e3) / 1e9

    # ---- roofline of the dominant kernel (algorithmic bytes / event time) ----
    peak, peak_src = measured_peaks()
    bound = "hbm"
    if args.workload in HOST_ARCS:
        # the arcs cross the host link every iteration: that link is the roof
        peak, peak_src, bound = round(host_link_gbs(dev), 1), "measured pinned H2D copy bandwidth (bench.py)", \
            "host-link"
    dom = max((k for k in kstats if kstats[k]["launches"] and k.startswith("mfl_")),
              key=lambda k: kstats[k]["ms"], default=None)
    roof = None
    if dom:
        s = kstats[dom]
        achieved = s["bytes"] / (s["ms"] / 1e3) / 1e9  # GB/s
        traffic = None
        tfile = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tfile):
            try:
                traffic = json.load(open(tfile)).get(args.workload, {}).get(dom)
            except (OSError, ValueError):
                traffic = None
        gceil = None
        gfile = os.path.join(ROOT, "profiles", "gather_ceilings.json")
        if os.path.exists(gfile):
            try:
                gceil = json.load(open(gfile)).get(args.workload)
            except (OSError, ValueError):
                gceil = None
        gath = s["arcs"] / (s["ms"] / 1e3) / 1e9  # one label gather per arc
        gb = 8 if variant == "llp" else 4
        label_mb = n * gb / 1e6
        roof = {"bound": bound, "kernel": dom, "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic, "peak_source": peak_src,
                "bytes_per_launch": s["bytes"] / s["launches"], "ms_per_launch": s["ms"] / s["launches"],
                "share_of_step": round(s["ms"] / sum(prof_ms), 3) if world == 1 else None,
                # the ceiling that actually binds: one random 4-B label gather per
                # arc costs a 32-B sector, measured by tools/ubench.py
                "gather_ceiling": {"achieved": round(gath, 1), "peak": gceil, "unit": "G label gathers/s",
                                   "frac": round(gath / gceil, 4) if gceil else None,
                                   "source": "profiles/gather_ceilings.json"},
                # SURVEY §8(d) "labels beyond L2" (TaoBao, R28): the label
                # gathers are HBM traffic too -- 4 B per gathered label (8 B:
                # LLP's (label, V) pairs), credited here as a second figure
                "with_gathers": ({"achieved": round((s["bytes"] + gb * s["arcs"]) / (s["ms"] / 1e3) / 1e9, 1),
                                  "frac": round((s["bytes"] + gb * s["arcs"]) / (s["ms"] / 1e3) / 1e9 / peak, 4),
                                  "bytes_per_gather": gb,
                                  "why": f"label array {label_mb:.0f} MB exceeds the 126 MB L2"}
                                 if label_mb > 126 else None),
                "kernel_timing": f"{kprof_steps} profiled steps with the class kernels serialised (CUDA events per "
                                 f"launch; {sum(prof_ms) / kprof_steps:.3f} ms/step serialised vs the timed region's "
                                 f"concurrent steps)",
                "kernels": {k: {"ms": round(v["ms"] / kprof_steps, 4), "launches": v["launches"] // kprof_steps,
                                "Garcs_s": round(v["arcs"] / max(v["ms"], 1e-9) / 1e6, 1),
                                "GBps_alg": round(v["bytes"] / max(v["ms"], 1e-9) / 1e6, 1)}
                            for k, v in kstats.items() if v["launches"]}}

    out = None
    if rank == 0:
        st = g.iter_stats()
        # whole-iteration roofline (SURVEY §8(d) model incl. 4n label first touch)
        it_bytes = [4.0 * s["active_arcs"] + 8.0 * s["active_vertices"] + 4.0 * n + 4.0 * s["changed"] for s in st]
        it1 = st[0] if st else None
        if roof is not None and st:
            # every iteration of the last timed run against the same HBM peak:
            # B_t (4 arcs + 8 vertices + 4n + 4 changed) / t_iter
            roof["per_iteration"] = [
                {"t": i + 1, "ms": round(x["ms"], 4), "active_arcs": x["active_arcs"],
                 "bytes": int(b), "gbps": round(b / (x["ms"] / 1e3) / 1e9, 1),
                 "frac": round(b / (x["ms"] / 1e3) / 1e9 / peak, 4),
                 "gteps": round(x["active_arcs"] / (x["ms"] / 1e3) / 1e9, 2)}
                for i, (x, b) in enumerate(zip(st, it_bytes)) if x["ms"] > 0]
            tot_ms = sum(x["ms"] for x in st)
            roof["whole_run"] = {"bytes": int(sum(it_bytes)), "ms": round(tot_ms, 4),
                                 "frac": round(sum(it_bytes) / (tot_ms / 1e3) / 1e9 / peak, 4) if tot_ms else None}
        out = {
            "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic",
            "config": {"workload": args.workload, "generator": spec, "variant": variant, "gamma": gamma,
                       "max_iters": max_iters, "n": n, "arcs": nnz, "parallelism": f"vertex-range x{world}",
                       "l2": f"inputs larger than L2 ({4 * nnz / 1e9:.2f} GB of arcs) and a 256 MB L2 flush "
                             "before every step",
                       "graph_gen_s": round(t_gen, 2), "bins": info["bins"], "max_degree": info["max_degree"]},
            "iterations": iters, "stop_reason": glp.STOP_NAMES[infos[-1].stop_reason],
            "time_to_converge_ms": round(ms_per_step, 4),
            "iteration_ms": [round(s["ms"], 4) for s in st],
            "iteration_active_arcs": [s["active_arcs"] for s in st],
            "iteration1_gteps": round(nnz / (it1["ms"] / 1e3) / 1e9, 2) if it1 else None,
            "iteration1_hbm_frac": round(it_bytes[0] / (it1["ms"] / 1e3) / 1e9 / peak, 4) if it1 else None,
            "nnz_x_iterations_gteps": round(nnz_iters, 3),
            "scanned_arcs_per_step": int(scanned / args.steps),
            "roofline": roof,
            "gpu_launches": int(sum(i.kernel_launches for i in infos)),
            "clocks": clk.summary(),
        }
    if e2e is not None:
        out["e2e"] = e2e
    # ---- CPU baseline: the oracle on a bounded sample of the same workload ----
    if rank == 0 and world == 1 and not args.no_cpu:
        csr_cpu = csr.to("cpu")
        samp_iters = 1 if nnz > 50_000_000 else max_iters
        v, cores, sec, its = cpu_reference(csr_cpu, variant, seeds, gamma, samp_iters, reps=1, weights=wts)
        out["cpu_baseline"] = {"value": round(v, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
                               "cpu_model": cpu_model(),
                               "sample": f"{args.workload}: first {its} LP iteration(s) from PickLabel, "
                                         f"oracle/glp_oracle.c OpenMP over {cores} threads, {sec:.1f} s "
                                         "(the oracle scans every arc each iteration)",
                               "sequential": cpu_sequential(csr_cpu, variant, seeds, gamma)
                               if wts is None and variant != "slp" else None}
    if rank == 0:
        print(json.dumps(out), flush=True)
    g.close()
    if world > 1:
        dist.destroy_process_group()


def bench_reference(args):
    """--impl reference: the CPU oracle (as it stands) on the same workload."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch
    spec, variant, max_iters, gamma = WORKLOADS[args.workload]
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    csr, seeds = make_graph(spec, dev)
    wts = workload_weights(args.workload, csr)
    wts = None if wts is None else wts.cpu()
    csr_cpu = csr.to("cpu")
    del csr
    seeds = None if seeds is None else seeds.cpu()
    # each step = one whole run of the workload (same config as the GPU arm)
    # when K+W of them fit the budget, else the first `samp` iterations
    _, _, probe_s, probe_it = cpu_reference(csr_cpu, variant, seeds, gamma, 1, reps=1, weights=wts)
    budget_s = float(os.environ.get("GLP_REF_BUDGET_S", "200"))
    per_it = probe_s / max(probe_it, 1)
    samp = max_iters if per_it * max_iters * (args.steps + args.warmup) <= budget_s else \
        max(1, int(budget_s / (per_it * (args.steps + args.warmup))))
    samp = min(samp, max_iters)
    v, cores, sec, its = cpu_reference(csr_cpu, variant, seeds, gamma, samp, reps=args.steps, warmup=args.warmup,
                                       weights=wts)
    same = samp == max_iters
    out = {"metric": METRIC, "value": round(v, 4), "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(sec * 1e3, 2), "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic", "impl": "reference",
           "config": {"workload": args.workload, "generator": spec, "variant": variant, "gamma": gamma,
                      "max_iters": max_iters, "n": csr_cpu.n, "arcs": csr_cpu.nnz, "same_config": same},
           "cpu_baseline": {"value": round(v, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
                            "cpu_model": cpu_model(),
                            "sample": (f"each step = one whole run of {args.workload} (stop rule, <= {max_iters} "
                                       "iterations)" if same else
                                       f"each step = first {samp} LP iteration(s) of {args.workload} from "
                                       "PickLabel") + f"; {its} iterations timed over {args.steps} steps"},
           "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="glp", choices=["glp", "reference"])
    ap.add_argument("--workload", default="rmat24", choices=sorted(WORKLOADS))
    ap.add_argument("--max-iters", type=int, default=None)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    args = ap.parse_args()
    if args.impl == "reference":
        bench_reference(args)
    else:
        bench_gpu(args)


if __name__ == "__main__":
    main()
