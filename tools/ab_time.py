"""A/B timing of one libglp build (GLP_LIB=build/<variant>.so) on the GPU box.

  python tools/ab_time.py WORKLOAD [REPS]     (WORKLOAD: a bench.py workload)

Runs REPS complete runs (L2 flushed before each, concurrent class kernels as
in bench.py's timed region), prints one JSON line: median/min ms per run,
per-iteration ms of the median run, and a label checksum (variants must agree).
"""
import hashlib
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_sigmod_yelhls21_b200 as glp  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "rmat24"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
kw = json.loads(os.environ.get("GLP_AB_KW", "{}"))  # extra glp_run params (A/B of run modes)
csr, seeds = bench.make_graph(spec, "cuda")
torch.cuda.synchronize()
torch.cuda.empty_cache()
g = glp.Graph(csr, weights=bench.workload_weights(wl, csr))
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")
stream = torch.cuda.current_stream()
for _ in range(3):
    g.run(variant, max_iters, seeds, gamma=gamma, **kw)
ms, its, shas = [], [], set()
for _ in range(reps):
    flush.fill_(1)
    info = g.run(variant, max_iters, seeds, gamma=gamma, **kw)
    ms.append(info.elapsed_ms)
    its.append([round(s["ms"], 3) for s in g.iter_stats()])
    shas.add(hashlib.sha1(g.labels("cpu").numpy().tobytes()).hexdigest()[:12])
lab = g.labels("cpu").numpy()
cs = csr.col_idx[: 1 << 28]  # bounded (R28 has 8.5e9 arcs)
w = (torch.arange(cs.numel(), device="cuda", dtype=torch.int64) % 1000003) + 1
graph_sum = int((cs.to(torch.int64) * w).sum()) ^ int(csr.row_offsets.sum())
del cs, w
med = statistics.median(ms)
i = ms.index(sorted(ms)[len(ms) // 2])
print(json.dumps({"lib": os.environ.get("GLP_LIB", "in-tree"), "kw": kw, "workload": wl, "median_ms": round(med, 3),
                  "min_ms": round(min(ms), 3), "iterations": info.iterations, "iter_ms": its[i],
                  "labels_sha": hashlib.sha1(lab.tobytes()).hexdigest()[:12], "distinct_runs": len(shas),
                  "graph_sum": graph_sum}), flush=True)
