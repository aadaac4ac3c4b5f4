"""§8(f)3 SLP on the GPU (speaker-listener LP [P:120]; the classic MFL
kernels count the speakers, k_slp_listen_speak updates the candidates) vs the
SLP oracle: every vertex's K candidate slots (labels and counts) and the
speakers, bit for bit."""
import numpy as np
import pytest

import oracle
from glp_inputs import graphs

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


@pytest.mark.parametrize("K,r", [(5, 0.0), (5, 0.1), (1, 0.0), (3, 0.3), (16, 0.05)])
def test_slp_matches_oracle(K, r):
    csr = graphs.rmat(14, seed=12)
    T = 20
    ml, mc, sp = oracle.run_slp(csr, K=K, r=r, max_iters=T, threads=8)
    with glp.Graph(csr.to("cuda")) as g:
        info = g.run("slp", T, slp_max_labels=K, slp_threshold=r)
        assert info.iterations == T and info.stop_reason == 0
        lab = g.labels("cpu").numpy()
        gl, gc = g.slp_memory(K)
    assert (lab == sp).all()
    assert (gl.numpy() == ml).all() and (gc.numpy() == mc).all()


def test_slp_sbm_and_local_group():
    from paper_conf_sigmod_yelhls21_b200.dist import LocalGroup
    csr = graphs.sbm(n=20_010, k=30, m=200_000, mu=0.2, seed=4)
    ml, mc, sp = oracle.run_slp(csr, K=5, r=0.05, max_iters=20, threads=8)
    with LocalGroup(csr.to("cuda"), 3) as grp:
        grp.run("slp", 20, slp_max_labels=5, slp_threshold=0.05)
        for r in range(3):
            assert (grp.labels(r).numpy() == sp).all()
        b = grp.bounds
        for r in range(3):
            gl, gc = grp.graphs[r].slp_memory(5, b[r + 1] - b[r])
            assert (gl.numpy() == ml[b[r]:b[r + 1]]).all() and (gc.numpy() == mc[b[r]:b[r + 1]]).all()


def test_slp_errors():
    csr = graphs.karate().to("cuda")
    with glp.Graph(csr) as g:
        g.run("classic", 5)
        with pytest.raises(glp.GlpError) as e:
            g.slp_memory(5)
        assert e.value.status == 7
        with pytest.raises(glp.GlpError):
            g.run("slp", 5, slp_max_labels=17)
