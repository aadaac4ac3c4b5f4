"""CUDA path (through the C ABI) vs the CPU oracle, element by element.

Integer variants (CLASSIC, SEEDED) must be bit-exact; LLP is computed in
double on both sides with the same operation order, so it is held to
bit-exact labels too (north_star floor: modularity within 1e-9 and >= 99.99 %
label agreement, checked as well).
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from glp_inputs import graphs
from glp_inputs.csr import CSR, from_arrays, from_edges

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


def gpu(csr, variant=0, max_iters=20, seeds=None, gamma=0.0, frontier=-1, on_device=True,
        stop_on_2cycle=True, dense_divisor=0, debug_pred_cap=0):
    c = csr.to("cuda") if on_device else csr
    with glp.Graph(c) as g:
        info = g.run(variant, max_iters, seeds, gamma=gamma, frontier=frontier,
                     stop_on_2cycle=stop_on_2cycle, dense_divisor=dense_divisor,
                     debug_pred_cap=debug_pred_cap)
        lab = g.labels("cpu").numpy().copy()
        st = g.iter_stats()
    return lab, info, st


def assert_same_run(csr, variant=0, max_iters=20, seeds=None, gamma=0.0, frontier=-1, **kw):
    ref = oracle.run(csr, variant, max_iters, seeds=None if seeds is None else np.asarray(seeds),
                     gamma=gamma, threads=8)
    lab, info, st = gpu(csr, variant, max_iters, seeds, gamma, frontier, **kw)
    assert info.iterations == ref.iterations, (info, ref)
    assert info.stop_reason == ref.stop_reason
    assert [s["changed"] for s in st] == list(ref.changed)
    mism = np.flatnonzero(lab != ref.labels)
    assert mism.size == 0, f"{mism.size} labels differ, first {mism[:10]}"
    return ref, lab, info, st


# --------------------------------------------------------------------------- small, per iteration
def test_bowtie_golden_trajectories(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "bowtie.json")))
    csr = from_arrays(g["graph"]["n"], g["graph"]["row_offsets"], g["graph"]["col_idx"], symmetric=True)
    for case, variant in [("classic", 0), ("llp_gamma_1", 2), ("seeded_4", 1), ("seeded_1_4", 1)]:
        exp = g[case]
        for t, row in enumerate(exp["trajectory"], start=1):
            lab, info, _ = gpu(csr, variant, t, exp.get("seeds"), exp.get("gamma", 0.0))
            assert lab.tolist() == row, (case, t)
        lab, info, st = gpu(csr, variant, 20, exp.get("seeds"), exp.get("gamma", 0.0))
        assert info.iterations == exp["iterations"] and info.stop_reason == exp["stop_reason"]
        assert [s["changed"] for s in st] == exp["changed"]


def test_karate():
    ref, lab, info, st = assert_same_run(graphs.karate())
    assert info.iterations == 11 and (lab == 0).all()


@pytest.mark.parametrize("name", ["k2", "star", "k34", "p6", "cliques", "empty", "single"])
def test_small_shapes(name):
    csr = {"k2": graphs.path(2), "star": graphs.star(40), "k34": graphs.complete_bipartite(3, 4),
           "p6": graphs.path(6), "cliques": graphs.cliques([3, 5, 40, 33, 300]), "empty": graphs.empty(7),
           "single": graphs.empty(1)}[name]
    for variant, gamma in [(0, 0.0), (2, 1.0), (2, 0.5)]:
        assert_same_run(csr, variant, 20, gamma=gamma)


def test_zero_vertices_and_zero_iters():
    z = graphs.empty(0)
    lab, info, st = gpu(z, 0, 5)
    assert lab.size == 0 and info.iterations == 1 and info.stop_reason == 1
    lab, info, st = gpu(graphs.karate(), 0, 0)
    assert info.iterations == 0 and lab.tolist() == list(range(34))


@pytest.mark.parametrize("seed", range(40))
def test_random_tiny_all_variants(seed):
    n = 5 + seed % 37
    csr = graphs.gnp(n, 0.05 + (seed % 7) * 0.08, seed=seed)
    seeds = [v for v in range(n) if (v * 13 + seed) % 9 == 0]
    assert_same_run(csr, 0, 30)
    assert_same_run(csr, 1, 30, seeds=seeds)
    for gamma in (0.0, 0.25, 1.0, 0.3):
        assert_same_run(csr, 2, 12, gamma=gamma)


def test_per_iteration_trace_rmat():
    csr = graphs.rmat(12, seed=9)
    ref = oracle.run(csr, 0, 12, trace=True, threads=8)
    for t in range(1, ref.iterations + 1):
        lab, info, _ = gpu(csr, 0, t)
        assert (lab == ref.trace[t - 1]).all(), t


# --------------------------------------------------------------------------- degree bins
def _degree_mix(degrees, seed=0, extra_pairs=0):
    """Vertex i (i < len(degrees)) gets exactly degrees[i] distinct leaf
    neighbours in its own leaf pool; leaves are then cross-linked at random so
    labels repeat with varying multiplicities."""
    src, dst = [], []
    base = len(degrees)
    for i, d in enumerate(degrees):
        leaves = np.arange(base, base + d)
        src.append(np.full(d, i))
        dst.append(leaves)
        base += d
    n = base
    g = np.random.default_rng(seed)
    if extra_pairs:
        a = g.integers(len(degrees), n, extra_pairs)
        b = g.integers(len(degrees), n, extra_pairs)
        src.append(a)
        dst.append(b)
    s = torch.from_numpy(np.concatenate(src).astype(np.int64))
    d = torch.from_numpy(np.concatenate(dst).astype(np.int64))
    return from_edges(n, s, d, "degmix")


@pytest.mark.parametrize("degrees", [
    [1, 2, 31, 32, 33, 34],
    [255, 256, 257, 258, 511],
    [4095, 4096, 4097, 8000],
    [30000],                 # > smem table: overflow -> global recount
    [70000, 5, 300, 5000],
])
def test_bin_boundaries(degrees):
    csr = _degree_mix(degrees, seed=len(degrees), extra_pairs=sum(degrees) // 2)
    assert_same_run(csr, 0, 15)
    assert_same_run(csr, 2, 6, gamma=0.5)
    assert_same_run(csr, 1, 15, seeds=[0, len(degrees) + 3])


@pytest.mark.parametrize("cap", [1, 40, 300])
def test_requeue_paths_exact(cap):
    """Under-predicted distinct counts force every overflow / re-queue path
    (W -> M -> L, partition retries); results must not change."""
    for csr in [_degree_mix([70000, 20000, 5000, 3000, 1500, 600, 300, 100, 40], seed=3, extra_pairs=60000),
                graphs.rmat(14, seed=5)]:
        assert_same_run(csr, 0, 12, debug_pred_cap=cap)
        assert_same_run(csr, 2, 5, gamma=0.25, debug_pred_cap=cap)


def test_giant_rows_epoch_wrap():
    """Giant rows (deg > 65536) use epoch-tagged global tables that are only
    cleared when the 8-bit epoch wraps: run past several wraps."""
    csr = graphs.star(70000)
    ref = oracle.run(csr, 0, 600, stop_on_2cycle=False)
    lab, info, st = gpu(csr, 0, 600, stop_on_2cycle=False)
    assert info.iterations == 600 and (lab == ref.labels).all()
    csr = _degree_mix([200000, 90000, 70000, 66000, 3000], seed=5, extra_pairs=300000)
    for _ in range(2):
        assert_same_run(csr, 0, 20)
        assert_same_run(csr, 1, 20, seeds=[0, 1, 7, 400000])
        assert_same_run(csr, 2, 6, gamma=1.0)


def _perturb_rows(csr, mode, seed=0):
    """Same graph, different arc order inside rows: 'shuffle' every row, or
    'tail' = swap the last two arcs of every row (sorted until the very end)."""
    off, col = csr.numpy()
    col = col.copy()
    g = np.random.default_rng(seed)
    for v in range(csr.n):
        a, b = off[v], off[v + 1]
        if b - a < 2:
            continue
        if mode == "shuffle":
            col[a:b] = g.permutation(col[a:b])
        else:
            col[b - 2], col[b - 1] = col[b - 1], col[b - 2]
    return from_arrays(csr.n, off, col, symmetric=csr.symmetric)


@pytest.mark.parametrize("mode", ["shuffle", "tail"])
def test_unsorted_rows_sorted_fast_path(mode):
    """The sorted-row fast path (t = 1) must agree with the table path on any
    arc order, including rows that stop being sorted in their last round."""
    base = _degree_mix([70000, 9000, 3000, 1500, 600, 300, 130, 40], seed=2, extra_pairs=40000)
    for csr in [base, graphs.rmat(13, seed=3)]:
        pert = _perturb_rows(csr, mode)
        for variant, gamma in [(0, 0.0), (2, 0.5)]:
            a = gpu(csr, variant, 6, gamma=gamma)
            b = gpu(pert, variant, 6, gamma=gamma)
            assert (a[0] == b[0]).all()
            ref = oracle.run(pert, variant, 6, gamma=gamma, threads=8)
            assert (b[0] == ref.labels).all()


def test_hub_with_few_labels_and_ties():
    # a hub whose neighbours carry a handful of labels: hot keys (warp
    # aggregation) and an exact tie resolved to the smaller label
    n = 20001
    src = torch.zeros(20000, dtype=torch.int64)
    dst = torch.arange(1, 20001, dtype=torch.int64)
    # leaves form 4 cliques-of-paths so their labels collapse to 4 values
    grp = (dst - 1) % 4
    s2 = dst[4:]
    d2 = dst[:-4]
    csr = from_edges(n, torch.cat([src, s2]), torch.cat([dst, d2]))
    del grp
    assert_same_run(csr, 0, 20)
    assert_same_run(csr, 2, 8, gamma=1.0)


# --------------------------------------------------------------------------- graph families
@pytest.mark.parametrize("scale", [10, 14, 16])
def test_rmat_classic(scale):
    assert_same_run(graphs.rmat(scale, seed=scale), 0, 20)


def test_rmat_llp_thrash_bitexact():
    csr = graphs.rmat(14, seed=2)
    for gamma in (1.0, 0.125, 0.37, 8.0):
        ref, lab, info, st = assert_same_run(csr, 2, 10, gamma=gamma)
        q_ref = oracle.modularity(csr, ref.labels)
        q_gpu = oracle.modularity(csr, lab)
        assert abs(q_ref - q_gpu) <= 1e-9
        assert (lab == ref.labels).mean() >= 0.9999


def test_sbm_classic():
    assert_same_run(graphs.sbm(n=100_000, k=100, m=2_000_000, seed=5), 0, 30)


def test_taobao_seeded_small():
    csr, seeds = graphs.taobao(users=200_000, items=50_000, pairs=2_000_000, rings=200, seed=7)
    assert_same_run(csr, 1, 30, seeds=seeds)


# --------------------------------------------------------------------------- frontier / modes
def test_frontier_equals_full_sweep():
    for csr in [graphs.rmat(14, seed=4), graphs.sbm(n=50_000, k=50, m=500_000, seed=3)]:
        a = gpu(csr, 0, 30, frontier=0)
        b = gpu(csr, 0, 30, frontier=1, dense_divisor=1)  # sparse unless every arc changed
        c = gpu(csr, 0, 30)
        assert (a[0] == b[0]).all() and (a[0] == c[0]).all()
        assert a[1].iterations == b[1].iterations == c[1].iterations
        assert any(not s["dense"] for s in b[2][1:])
        # the sparse iterations really skip work
        assert sum(s["active_arcs"] for s in b[2]) < sum(s["active_arcs"] for s in a[2])


def test_seeded_frontier_and_bfs_reach():
    csr, seeds = graphs.taobao(users=40_000, items=10_000, pairs=200_000, rings=40, seed=5)
    a = gpu(csr, 1, 40, seeds, frontier=0)
    b = gpu(csr, 1, 40, seeds)
    assert (a[0] == b[0]).all()
    s = seeds.numpy()
    assert (b[0][s] == s).all()


def test_host_and_device_inputs_identical():
    csr = graphs.rmat(13, seed=11)
    a = gpu(csr, 0, 20, on_device=True)
    b = gpu(csr, 0, 20, on_device=False)
    assert (a[0] == b[0]).all()


def test_deterministic_repeat():
    csr = graphs.rmat(15, seed=6)
    c = csr.to("cuda")
    with glp.Graph(c) as g:
        g.run("classic", 20)
        x = g.labels("cpu").clone()
        g.run("llp", 6, gamma=1.0)
        g.run("classic", 20)
        y = g.labels("cpu").clone()
    assert torch.equal(x, y)


def test_no_2cycle_stop():
    csr = graphs.path(2)
    ref = oracle.run(csr, 0, 9, stop_on_2cycle=False)
    lab, info, st = gpu(csr, 0, 9, stop_on_2cycle=False)
    assert info.iterations == 9 and info.stop_reason == 0 and (lab == ref.labels).all()


# --------------------------------------------------------------------------- errors
def test_error_codes():
    csr = graphs.karate().to("cuda")
    with glp.Graph(csr) as g:
        with pytest.raises(glp.GlpError) as e:
            g.labels()
        assert e.value.status == 7
        for kw, st in [(dict(max_iters=-1), 1), (dict(variant="classic", seeds=[1]), 1),
                       (dict(variant="llp", gamma=float("nan")), 1), (dict(variant="llp", gamma=-1.0), 1),
                       (dict(variant="llp", frontier=1), 1), (dict(variant="seeded", seeds=[99]), 1)]:
            with pytest.raises(glp.GlpError) as e:
                args = dict(variant="classic", max_iters=5)
                args.update(kw)
                v = args.pop("variant")
                m = args.pop("max_iters")
                g.run(v, m, **args)
            assert e.value.status == st, kw
    bad = CSR(3, torch.tensor([0, 1, 2, 3], dtype=torch.int64, device="cuda"),
              torch.tensor([1, 0, 7], dtype=torch.int32, device="cuda"))
    with pytest.raises(glp.GlpError) as e:
        glp.Graph(bad)
    assert e.value.status == 2
    bad = CSR(3, torch.tensor([0, 2, 1, 3], dtype=torch.int64), torch.tensor([1, 0, 1], dtype=torch.int32))
    with pytest.raises(glp.GlpError) as e:
        glp.Graph(bad)
    assert e.value.status == 2


def test_nccl_exchange_path_single_rank():
    """A one-rank NCCL communicator drives the multi-GPU exchange code
    (all-gather of labels, counter all-reduce, frontier-mark reduce-scatter)
    on one GPU; results must equal the single-GPU path and the oracle."""
    for csr, variant, seeds, gamma in [(graphs.rmat(14, seed=8), "classic", None, 0.0),
                                       (graphs.rmat(13, seed=9), "llp", None, 1.0)]:
        uid = glp.glp_nccl_unique_id()
        c = csr.to("cuda")
        with glp.Graph(c, rank=0, nranks=1, nccl_unique_id=uid, device=0) as g:
            info = g.run(variant, 12, seeds, gamma=gamma)
            lab = g.labels("cpu").numpy()
        ref = oracle.run(csr, glp.VARIANTS[variant], 12, gamma=gamma, threads=8)
        assert info.iterations == ref.iterations and (lab == ref.labels).all()
        if variant == "classic":  # the NCCL sparse exchange calls (§8(f)1), one rank
            with glp.Graph(c, rank=0, nranks=1, nccl_unique_id=glp.glp_nccl_unique_id(), device=0) as g:
                info = g.run(variant, 12, seeds, sparse_exchange=1)
                lab = g.labels("cpu").numpy()
                assert {s["exchange"] for s in g.iter_stats()} == {2}
            assert info.iterations == ref.iterations and (lab == ref.labels).all()
    csr, seeds = graphs.taobao(users=40_000, items=10_000, pairs=200_000, rings=40, seed=5)
    uid = glp.glp_nccl_unique_id()
    with glp.Graph(csr.to("cuda"), rank=0, nranks=1, nccl_unique_id=uid, device=0) as g:
        info = g.run("seeded", 30, seeds.numpy())
        lab = g.labels("cpu").numpy()
    ref = oracle.run(csr, oracle.SEEDED, 30, seeds=seeds.numpy(), threads=8)
    assert info.iterations == ref.iterations and (lab == ref.labels).all()


@pytest.mark.parametrize("env", [{"GLP_NO_VL": "1"}, {"GLP_SERIAL": "1"}, {"GLP_DEVICE_LOOP": "1"},
                                 {"GLP_NO_MONO": "1"}])
def test_alternate_execution_modes(env, monkeypatch):
    """The A/B switches read at graph create (LLP without the interleaved
    label/V array, serialised class kernels) give the same exact runs."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    csr = graphs.rmat(13, seed=4)
    assert_same_run(csr, 0, 20)
    for gamma in (1.0, 0.37):
        assert_same_run(csr, 2, 8, gamma=gamma)
    tb, seeds = graphs.taobao(users=40_000, items=10_000, pairs=200_000, rings=40, seed=5)
    assert_same_run(tb, 1, 30, seeds=seeds.numpy())  # sparse frontier iterations
    assert_same_run(graphs.karate(), 0, 20)


def _label_part(lab, nparts):
    """Host copy of the L kernel's label-partition hash (mfl_kernels.cuh
    label_part), used only to build inputs that load chosen parts."""
    h = (lab.astype(np.uint64) * np.uint64(0x85EBCA77) + np.uint64(0x165667B1)) & np.uint64(0xFFFFFFFF)
    return ((h * np.uint64(nparts)) >> np.uint64(32)).astype(np.int64)


def _hub_distinct_t2(labels_of_leaves):
    """A hub whose leaf i also touches a private vertex p_i with a smaller id:
    at t = 1 leaf i takes label p_i, so at t = 2 the hub sees one distinct
    label per arc (its row took the sorted fast path at t = 1, so its
    distinct-count estimate is a fraction of its degree)."""
    p = np.asarray(labels_of_leaves, dtype=np.int64)
    n = int(p.max()) + 1 + p.size + 1
    used = np.zeros(n, dtype=bool)
    used[p] = True
    used[n - 1] = True
    leaves = np.flatnonzero(~used)[: p.size]
    hub = n - 1
    src = np.concatenate([leaves, leaves])
    dst = np.concatenate([p, np.full(p.size, hub)])
    return from_edges(n, torch.from_numpy(src), torch.from_numpy(dst), "hub_t2")


@pytest.mark.parametrize("case", ["part1_heavy", "d20000", "d40000"])
def test_l_partition_retries_exact(case):
    """L rows whose t = 2 labels are all distinct: the filtered part counts,
    an overflow in the gather pass, an overflow in a later part (staged row,
    finer partitions) and the histogram path all give the oracle's labels."""
    if case == "part1_heavy":
        ids = np.arange(60000)
        part = _label_part(ids, 2)
        lab = np.concatenate([ids[part == 1][:10000], ids[part == 0][:500]])
    else:
        d = 20000 if case == "d20000" else 40000
        lab = np.random.default_rng(d).permutation(3 * d)[:d]
    csr = _hub_distinct_t2(np.sort(lab))
    assert_same_run(csr, 0, 6)
    assert_same_run(csr, 2, 4, gamma=0.5)
    assert_same_run(csr, 1, 6, seeds=[0, int(lab.min()), csr.n - 1])


# --------------------------------------------------------------------------- SEEDED presence filter
@pytest.mark.parametrize("case", ["taobao", "hubs", "rmat_few_seeds"])
def test_seeded_presence_filter_forced(case, monkeypatch):
    """GLP_LBITS=1 forces the SEEDED presence bitmap (normally only for label
    arrays larger than L2): labels and per-iteration changes stay those of the
    oracle through every row class (low, W pairs, W, M, L, giant)."""
    monkeypatch.setenv("GLP_LBITS", "1")
    if case == "taobao":
        csr, seeds = graphs.taobao(users=200_000, items=50_000, pairs=2_000_000, rings=200, seed=7)
    elif case == "hubs":
        csr = _degree_mix([3, 40, 70, 300, 3000, 9000, 70000], seed=4, extra_pairs=200_000)
        seeds = torch.tensor([0, 5, 17, 123, 4000], dtype=torch.int32)
    else:
        csr = graphs.rmat(15, seed=9)
        seeds = torch.tensor([1, 2, 3, 100, 2000, 30000], dtype=torch.int32)
    ref, lab, info, st = assert_same_run(csr, 1, 30, seeds=seeds)
    # the filter is on while at most half the vertices can be labelled
    assert info.iterations >= 2


@pytest.mark.parametrize("short", ["0", "1"])
def test_w_kernel_block_variants(short, monkeypatch):
    """The W kernel at 4 or 3 blocks/SM (GLP_W_SHORT forces the choice made
    from the graph's row lengths) gives the oracle's labels, on a graph with
    both 33-64-arc rows (pair path) and longer W rows."""
    monkeypatch.setenv("GLP_W_SHORT", short)
    assert_same_run(graphs.sbm(n=60_000, k=60, m=1_500_000, seed=9), 0, 30)
    assert_same_run(graphs.rmat(14, seed=6), 0, 20)
