"""§8(f)4 CPU-GPU hybrid mode ("one or multiple GPUs", graphs beyond device
memory [P:103]): the arc array lives in pinned, mapped host memory and every
iteration streams it over the host link.  Same kernels, same results: bit-exact
against the oracle."""
import numpy as np
import pytest

import oracle
from glp_inputs import graphs

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


def run_hybrid(csr, variant, max_iters, seeds=None, gamma=0.0):
    with glp.Graph(csr.to("cpu"), host_arcs=True) as g:
        info = g.run(variant, max_iters, seeds, gamma=gamma)
        lab = g.labels("cpu").numpy().copy()
        st = g.iter_stats()
    return lab, info, st


@pytest.mark.parametrize("variant", ["classic", "seeded", "llp"])
def test_hybrid_matches_oracle(variant):
    csr = graphs.rmat(14, seed=5)
    seeds = np.array([2, 99, 4000, 12345], dtype=np.int32) if variant == "seeded" else None
    gamma = 1.0 if variant == "llp" else 0.0
    mi = 10 if variant == "llp" else 20
    ref = oracle.run(csr, glp.VARIANTS[variant], mi, seeds=seeds, gamma=gamma, threads=8)
    lab, info, st = run_hybrid(csr, variant, mi, seeds, gamma)
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason)
    assert [s["changed"] for s in st] == list(ref.changed)
    assert (lab == ref.labels).all()


def test_hybrid_long_rows_and_pinned_input():
    """Giant / L rows, and a caller buffer that is already pinned."""
    csr = graphs.rmat(17, seed=2)
    ref = oracle.run(csr, oracle.CLASSIC, 20, threads=8)
    c = csr.to("cpu")
    c.col_idx = c.col_idx.pin_memory()
    with glp.Graph(c, host_arcs=True) as g:
        info = g.run("classic", 20)
        lab = g.labels("cpu").numpy()
    assert info.iterations == ref.iterations and (lab == ref.labels).all()


def test_hybrid_needs_host_csr():
    csr = graphs.karate().to("cuda")
    with pytest.raises(glp.GlpError) as e:
        glp.Graph(csr, host_arcs=True)
    assert e.value.status == 1
