"""Small runs of every kernel path, for compute-sanitizer (memcheck /
racecheck / synccheck / initcheck): classic, seeded (sparse frontier, long
push rows), LLP, forced W -> M -> L re-queues (debug_pred_cap), the L
partition passes, giant rows, weighted, hybrid (host arcs) and a 2-rank local
group; the W pair path (33-64-arc rows), the SEEDED presence filter and
the weighted low / warp / block / giant kernels.  Graphs are small so the
sanitizers finish in minutes."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigmod_yelhls21_b200 as glp
from paper_conf_sigmod_yelhls21_b200.dist import LocalGroup
from glp_inputs import graphs
from glp_inputs.csr import from_edges

which = sys.argv[1] if len(sys.argv) > 1 else "all"
csr = graphs.rmat(13, seed=3, device="cuda")
# hubs with > 65536 arcs (giant path) and distinct labels at t = 2 (L partitions)
g = np.random.default_rng(1)
n_priv = 80_000
leaves = n_priv + np.arange(n_priv)
src, dst = [np.arange(n_priv)], [leaves]
for h, d in enumerate([70000, 20000, 9000, 5000]):
    src.append(np.full(d, 2 * n_priv + h)); dst.append(g.choice(leaves, d, replace=False))
hubs = from_edges(2 * n_priv + 4, torch.from_numpy(np.concatenate(src)), torch.from_numpy(np.concatenate(dst))).to("cuda")
if which in ("all", "core"):
    with glp.Graph(csr) as G:
        print(G.run("classic", 20)); print(G.run("seeded", 20, [1, 50, 900]))
        print(G.run("llp", 5, gamma=1.0)); print(G.run("classic", 6, debug_pred_cap=8))
    with glp.Graph(hubs) as G:
        print(G.run("classic", 4)); print(G.run("llp", 3, gamma=0.5)); print(G.run("classic", 4, debug_pred_cap=16))
if which in ("all", "modes"):
    w = graphs.edge_weights(csr)
    with glp.Graph(csr, weights=w) as G:
        print(G.run("classic", 10))
    with glp.Graph(hubs, weights=graphs.edge_weights(hubs)) as G:  # partitioned weighted rows
        print(G.run("classic", 4))
    with glp.Graph(csr.to("cpu"), host_arcs=True) as G:
        print(G.run("classic", 10))
    with glp.Graph(csr) as G:
        print(G.run("slp", 8, slp_max_labels=5, slp_threshold=0.1))
    with glp.Graph(hubs) as G:  # HT + CMS, small HT: sketch, rescans, fallbacks
        print(G.run("classic", 4, tail_cms=True, cms_ht_slots=256))
    os.environ["GLP_LBITS"] = "1"  # SEEDED presence filter (normally only for label arrays beyond L2)
    with glp.Graph(csr) as G:
        print(G.run("seeded", 20, [1, 50, 900]))
    with glp.Graph(hubs) as G:
        print(G.run("seeded", 6, [0, 7, 2 * n_priv]))
    del os.environ["GLP_LBITS"]
    os.environ["GLP_DEVICE_LOOP"] = "1"
    with glp.Graph(csr) as G:
        print(G.run("classic", 20)); print(G.run("seeded", 20, [1, 50, 900]))
    del os.environ["GLP_DEVICE_LOOP"]
    with LocalGroup(csr, 2) as grp:
        print(grp.run("classic", 10)); print(grp.run("llp", 4, gamma=1.0))
        print(grp.run("classic", 10, sparse_exchange=1)); print(grp.run("seeded", 10, [1, 50, 900]))
print("sanitize run ok")
