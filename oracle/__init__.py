"""CPU oracle for GLP label propagation -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_sigmod_yelhls21_b200``) never imports it and shares no code with
it.  The arithmetic lives in ``glp_oracle.c`` (see its header for the paper
citations); this module only builds/loads it and marshals numpy arrays.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "glp_oracle.c")
LIB = os.path.join(HERE, "libglp_oracle.so")

CLASSIC, SEEDED, LLP = 0, 1, 2
STOP_MAX_ITERS, STOP_FIXED_POINT, STOP_TWO_CYCLE = 0, 1, 2

_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle (gcc, -ffp-contract=off, OpenMP)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
               "-shared", "-o", LIB, SRC]
        subprocess.check_call(cmd)
    return LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(LIB)
        P = ctypes.c_void_p
        lib.glp_oracle_run.restype = ctypes.c_int
        lib.glp_oracle_run.argtypes = [ctypes.c_int64, P, P, ctypes.c_int32, ctypes.c_int32, P,
                                       ctypes.c_int64, ctypes.c_double, ctypes.c_int32,
                                       ctypes.c_int32, P, P, P, P]
        lib.glp_oracle_step.restype = ctypes.c_int
        lib.glp_oracle_step.argtypes = [ctypes.c_int64, P, P, ctypes.c_int32, P, P, P, ctypes.c_double,
                                        ctypes.c_int64, ctypes.c_int64, P, ctypes.c_int32]
        lib.glp_oracle_run_w.restype = ctypes.c_int
        lib.glp_oracle_run_w.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, ctypes.c_int32, P,
                                         ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, P, P, P, P]
        lib.glp_oracle_slp.restype = ctypes.c_int
        lib.glp_oracle_slp.argtypes = [ctypes.c_int64, P, P, ctypes.c_int32, ctypes.c_double, ctypes.c_int32,
                                       ctypes.c_int32, P, P, P]
        lib.glp_oracle_modularity.restype = ctypes.c_double
        lib.glp_oracle_modularity.argtypes = [ctypes.c_int64, P, P, P]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _csr_np(csr_or_tuple):
    if isinstance(csr_or_tuple, tuple):
        n, off, col = csr_or_tuple
    else:
        n = csr_or_tuple.n
        off, col = csr_or_tuple.numpy()
    return (int(n), np.ascontiguousarray(off, dtype=np.int64),
            np.ascontiguousarray(col, dtype=np.int32))


class OracleResult:
    def __init__(self, labels, changed, iterations, reason, trace):
        self.labels = labels
        self.changed = changed
        self.iterations = iterations
        self.stop_reason = reason
        self.trace = trace  # [iterations, n] or None

    def __repr__(self):
        return (f"OracleResult(iterations={self.iterations}, stop_reason={self.stop_reason}, "
                f"changed={list(self.changed)})")


def run(csr, variant: int = CLASSIC, max_iters: int = 20, seeds=None, gamma: float = 0.0,
        stop_on_2cycle: bool = True, threads: int = 1, trace: bool = False) -> OracleResult:
    """Synchronous LP on the CPU (see glp_oracle.c for the definition)."""
    lib = _load()
    n, off, col = _csr_np(csr)
    labels = np.empty(max(n, 1), dtype=np.int32)
    changed = np.zeros(max(max_iters, 1), dtype=np.int64)
    tr = np.empty((max(max_iters, 1), max(n, 1)), dtype=np.int32) if trace else None
    info = np.zeros(2, dtype=np.int32)
    sd = None
    ns = 0
    if seeds is not None:
        sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.int32))
        ns = int(sd.size)
    rc = lib.glp_oracle_run(n, _ptr(off), _ptr(col), int(variant), int(max_iters), _ptr(sd), ns,
                            float(gamma), int(bool(stop_on_2cycle)), int(threads), _ptr(labels),
                            _ptr(changed), _ptr(tr), _ptr(info))
    if rc != 0:
        raise ValueError(f"glp_oracle_run failed rc={rc}")
    it = int(info[0])
    return OracleResult(labels[:n].copy(), changed[:it].copy(), it, int(info[1]),
                        None if tr is None else tr[:it, :n].copy())


def run_weighted(csr, weights, variant: int = CLASSIC, max_iters: int = 20, seeds=None,
                 stop_on_2cycle: bool = True, threads: int = 1, trace: bool = False) -> OracleResult:
    """Weighted LP (label frequency = sum of arc weights), CLASSIC/SEEDED."""
    lib = _load()
    n, off, col = _csr_np(csr)
    w = np.ascontiguousarray(np.asarray(weights.cpu().numpy() if hasattr(weights, "cpu") else weights,
                                        dtype=np.uint32))
    assert w.size == col.size
    labels = np.empty(max(n, 1), dtype=np.int32)
    changed = np.zeros(max(max_iters, 1), dtype=np.int64)
    tr = np.empty((max(max_iters, 1), max(n, 1)), dtype=np.int32) if trace else None
    info = np.zeros(2, dtype=np.int32)
    sd, ns = None, 0
    if seeds is not None:
        sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.int32))
        ns = int(sd.size)
    rc = lib.glp_oracle_run_w(n, _ptr(off), _ptr(col), _ptr(w), int(variant), int(max_iters), _ptr(sd), ns,
                              int(bool(stop_on_2cycle)), int(threads), _ptr(labels), _ptr(changed), _ptr(tr),
                              _ptr(info))
    if rc != 0:
        raise ValueError(f"glp_oracle_run_w failed rc={rc}")
    it = int(info[0])
    return OracleResult(labels[:n].copy(), changed[:it].copy(), it, int(info[1]),
                        None if tr is None else tr[:it, :n].copy())


def run_slp(csr, K: int = 5, r: float = 0.0, max_iters: int = 20, threads: int = 1):
    """Speaker-listener LP (see glp_oracle.c): returns (mem_labels [n, K],
    mem_counts [n, K], speakers [n])."""
    lib = _load()
    n, off, col = _csr_np(csr)
    ml = np.empty((max(n, 1), K), dtype=np.int32)
    mc = np.empty((max(n, 1), K), dtype=np.int32)
    sp = np.empty(max(n, 1), dtype=np.int32)
    rc = lib.glp_oracle_slp(n, _ptr(off), _ptr(col), int(K), float(r), int(max_iters), int(threads), _ptr(ml),
                            _ptr(mc), _ptr(sp))
    if rc != 0:
        raise ValueError(f"glp_oracle_slp failed rc={rc}")
    return ml[:n].copy(), mc[:n].copy(), sp[:n].copy()


def step(csr, variant: int, labels_prev, v_begin: int = 0, v_end=None, V=None, is_seed=None,
         gamma: float = 0.0, out=None, threads: int = 1) -> np.ndarray:
    """One synchronous iteration for rows [v_begin, v_end) (see glp_oracle.c)."""
    lib = _load()
    n, off, col = _csr_np(csr)
    v_end = n if v_end is None else v_end
    Lp = np.ascontiguousarray(labels_prev, dtype=np.int32)
    out = np.array(Lp, copy=True) if out is None else out
    Vh = None if V is None else np.ascontiguousarray(V, dtype=np.int32)
    sd = None if is_seed is None else np.ascontiguousarray(is_seed, dtype=np.uint8)
    rc = lib.glp_oracle_step(n, _ptr(off), _ptr(col), int(variant), _ptr(Lp), _ptr(Vh), _ptr(sd),
                             float(gamma), int(v_begin), int(v_end), _ptr(out), int(threads))
    if rc != 0:
        raise ValueError(f"glp_oracle_step failed rc={rc}")
    return out


def modularity(csr, labels) -> float:
    lib = _load()
    n, off, col = _csr_np(csr)
    lab = np.ascontiguousarray(np.asarray(labels, dtype=np.int32))
    return float(lib.glp_oracle_modularity(n, _ptr(off), _ptr(col), _ptr(lab)))


def init_labels(n: int, variant: int, seeds=None) -> np.ndarray:
    """L_0 as the oracle defines it (for tests that inspect t = 0)."""
    if variant == SEEDED:
        L = np.full(n, -1, dtype=np.int32)
        if seeds is not None and len(seeds):
            s = np.asarray(seeds, dtype=np.int64)
            L[s] = s
        return L
    return np.arange(n, dtype=np.int32)
