"""Parity at BASELINE.json's full sizes, in the configuration bench.py times.

The CPU oracle (OpenMP over the host cores) recomputes the same runs; labels
must match bit-exactly (CLASSIC / SEEDED), and LLP is held to bit-exact too
(north_star floor: modularity within 1e-9, >= 99.99 % agreement).
"""
import os

import numpy as np
import pytest
import torch

import oracle
from glp_inputs import graphs

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")
THREADS = os.cpu_count() or 8


@pytest.fixture(scope="module")
def rmat24():
    csr = graphs.rmat(24, seed=1, device="cuda")
    return csr, csr.to("cpu")


def _run(csr_dev, variant, max_iters, seeds=None, gamma=0.0):
    with glp.Graph(csr_dev) as g:
        info = g.run(variant, max_iters, seeds, gamma=gamma)
        lab = g.labels("cpu").numpy().copy()
        st = g.iter_stats()
    return lab, info, st


def test_rmat24_classic_to_convergence(rmat24):
    dev, cpu = rmat24
    lab, info, st = _run(dev, "classic", 20)
    ref = oracle.run(cpu, oracle.CLASSIC, 20, threads=THREADS)
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason)
    assert [s["changed"] for s in st] == list(ref.changed)
    assert (lab == ref.labels).all()


def test_rmat24_iteration1_closed_form(rmat24):
    """Unique labels: every count is 1, so L_1[v] = min N(v) (any size)."""
    dev, _ = rmat24
    lab, info, _ = _run(dev, "classic", 1)
    off = dev.row_offsets
    deg = off[1:] - off[:-1]
    rows = torch.repeat_interleave(torch.arange(dev.n, device="cuda"), deg)
    mins = torch.full((dev.n,), 2 ** 31 - 1, dtype=torch.int64, device="cuda")
    mins.scatter_reduce_(0, rows, dev.col_idx.to(torch.int64), reduce="amin")
    exp = torch.where(deg > 0, mins, torch.arange(dev.n, device="cuda")).cpu().numpy()
    assert (lab == exp).all()


def test_rmat24_llp_first_iterations(rmat24):
    dev, cpu = rmat24
    lab, info, _ = _run(dev, "llp", 4, gamma=1.0)
    ref = oracle.run(cpu, oracle.LLP, 4, gamma=1.0, threads=THREADS)
    assert info.iterations == ref.iterations
    agree = (lab == ref.labels).mean()
    assert agree >= 0.9999
    assert abs(oracle.modularity(cpu, lab) - oracle.modularity(cpu, ref.labels)) <= 1e-9
    assert (lab == ref.labels).all()


def test_sbm1m_classic_to_convergence():
    dev = graphs.sbm(device="cuda")
    cpu = dev.to("cpu")
    lab, info, st = _run(dev, "classic", 30)
    ref = oracle.run(cpu, oracle.CLASSIC, 30, threads=THREADS)
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason)
    assert (lab == ref.labels).all()


def test_taobao100m_seeded_first_iterations():
    dev, seeds = graphs.taobao(device="cuda")
    cpu = dev.to("cpu")
    s = seeds.cpu().numpy()
    lab, info, st = _run(dev, "seeded", 4, s)
    ref = oracle.run(cpu, oracle.SEEDED, 4, seeds=s, threads=THREADS)
    assert [x["changed"] for x in st] == list(ref.changed)
    assert (lab == ref.labels).all()
    assert (lab[s] == s).all()
