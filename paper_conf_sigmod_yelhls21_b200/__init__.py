"""B200-native GLP label propagation -- thin Python binding over libglp.so.

Argument marshalling only: every step of the LP iteration runs in the CUDA
kernels of ``csrc/`` behind the C ABI declared in ``include/glp.h``.  PyTorch
supplies device memory, streams and process groups.  There is no CPU fallback:
if ``libglp.so`` is missing or no B200 is visible the calls raise.

The function names mirror the C ABI (``glp_graph_create``, ``glp_run``,
``glp_labels_get`` ...); :class:`Graph` is a small convenience wrapper.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

from . import _build

HERE = os.path.dirname(os.path.abspath(__file__))
# GLP_LIB: load another in-tree build of the same library (kernel A/B experiments)
LIB_PATH = os.environ.get("GLP_LIB") or _build.LIB

CLASSIC, SEEDED, LLP, SLP = 0, 1, 2, 3
VARIANTS = {"classic": CLASSIC, "seeded": SEEDED, "llp": LLP, "slp": SLP}
STOP_MAX_ITERS, STOP_FIXED_POINT, STOP_TWO_CYCLE = 0, 1, 2
STOP_NAMES = {0: "max_iters", 1: "fixed_point", 2: "two_cycle"}
STATUS = {0: "GLP_OK", 1: "GLP_ERR_INVALID_ARGUMENT", 2: "GLP_ERR_INVALID_GRAPH",
          3: "GLP_ERR_OUT_OF_MEMORY", 4: "GLP_ERR_CUDA", 5: "GLP_ERR_NCCL",
          6: "GLP_ERR_UNSUPPORTED", 7: "GLP_ERR_STATE"}


class GlpError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


# ---------------------------------------------------------------- ctypes mirror of glp.h
class glp_csr(ctypes.Structure):
    _fields_ = [("n_global", ctypes.c_int64), ("v_begin", ctypes.c_int64), ("v_end", ctypes.c_int64),
                ("nnz_local", ctypes.c_int64), ("row_offsets", ctypes.c_void_p),
                ("col_idx", ctypes.c_void_p), ("on_device", ctypes.c_int32),
                ("symmetric", ctypes.c_int32), ("weights", ctypes.c_void_p)]


class glp_dist(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("nranks", ctypes.c_int32), ("device", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("cuda_stream", ctypes.c_void_p),
                ("local_group", ctypes.c_void_p)]


class glp_params(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("gamma", ctypes.c_double),
                ("frontier", ctypes.c_int32), ("stop_on_2cycle", ctypes.c_int32),
                ("validate", ctypes.c_int32), ("profile", ctypes.c_int32),
                ("dense_divisor", ctypes.c_int32), ("debug_pred_cap", ctypes.c_int32),
                ("llp_hist", ctypes.c_int32), ("host_arcs", ctypes.c_int32), ("tail_cms", ctypes.c_int32),
                ("cms_ht_slots", ctypes.c_int32), ("cms_depth", ctypes.c_int32),
                ("slp_max_labels", ctypes.c_int32), ("slp_threshold", ctypes.c_double),
                ("sparse_exchange", ctypes.c_int32)]


class glp_run_info(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_int32), ("stop_reason", ctypes.c_int32),
                ("changed_last", ctypes.c_int64), ("arcs_processed", ctypes.c_int64),
                ("elapsed_ms", ctypes.c_double), ("kernel_launches", ctypes.c_int64)]


class glp_iter_stat(ctypes.Structure):
    _fields_ = [("changed", ctypes.c_int64), ("d2", ctypes.c_int64),
                ("active_vertices", ctypes.c_int64), ("active_arcs", ctypes.c_int64),
                ("dense", ctypes.c_int32), ("exchange", ctypes.c_int32), ("ms", ctypes.c_double),
                ("cms_rows", ctypes.c_int64), ("cms_rescans", ctypes.c_int64), ("cms_fallbacks", ctypes.c_int64)]


class glp_kernel_stat(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("launches", ctypes.c_int64), ("ms", ctypes.c_double),
                ("bytes", ctypes.c_double), ("arcs", ctypes.c_double)]


EXPORTS = ["glp_nccl_unique_id", "glp_partition", "glp_graph_create", "glp_run", "glp_labels_get",
           "glp_iter_stats", "glp_kernel_stats", "glp_graph_info", "glp_graph_destroy",
           "glp_local_group_create", "glp_local_group_destroy", "glp_struct_sizes", "glp_slp_memory_get",
           "glp_last_error", "glp_version"]

_lib = None


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libglp.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"libglp.so not found at {path}; run __graft_entry__.build() "
                           "(there is no CPU fallback)")
    lib = ctypes.CDLL(path)
    P = ctypes.c_void_p
    I32, I64 = ctypes.c_int32, ctypes.c_int64
    sig = {
        "glp_nccl_unique_id": [P],
        "glp_partition": [P, I64, I32, I32, P],
        "glp_graph_create": [P, P, P, P],
        "glp_run": [P, I32, I32, P, I64, P, P],
        "glp_labels_get": [P, P, I64, I32],
        "glp_iter_stats": [P, P, I32, P],
        "glp_kernel_stats": [P, P, I32, P],
        "glp_graph_info": [P, P, I32],
        "glp_graph_destroy": [P],
        "glp_local_group_create": [I32, P],
        "glp_local_group_destroy": [P],
        "glp_struct_sizes": [P, I32],
        "glp_slp_memory_get": [P, P, P, I64, I32],
    }
    for name, args in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = ctypes.c_int
    lib.glp_last_error.restype = ctypes.c_char_p
    lib.glp_last_error.argtypes = []
    lib.glp_version.restype = ctypes.c_char_p
    lib.glp_version.argtypes = []
    _lib = lib
    return lib


def _check(st: int):
    if st != 0:
        raise GlpError(st, load_library().glp_last_error().decode(errors="replace"))


def make_params(gamma: float = 0.0, frontier: int = -1, stop_on_2cycle: bool = True,
                validate: bool = True, profile: bool = False, dense_divisor: int = 0,
                debug_pred_cap: int = 0, llp_hist: int = 0, host_arcs: bool = False, tail_cms: bool = False,
                cms_ht_slots: int = 0, cms_depth: int = 0, sparse_exchange: int = -1, slp_max_labels: int = 0,
                slp_threshold: float = 0.0) -> glp_params:
    p = glp_params()
    p.struct_size = ctypes.sizeof(glp_params)
    p.gamma = float(gamma)
    p.frontier = int(frontier)
    p.stop_on_2cycle = int(bool(stop_on_2cycle))
    p.validate = int(bool(validate))
    p.profile = int(bool(profile))
    p.dense_divisor = int(dense_divisor)
    p.debug_pred_cap = int(debug_pred_cap)
    p.llp_hist = int(llp_hist)
    p.host_arcs = int(bool(host_arcs))
    p.tail_cms = int(bool(tail_cms))
    p.cms_ht_slots = int(cms_ht_slots)
    p.cms_depth = int(cms_depth)
    p.sparse_exchange = int(sparse_exchange)
    p.slp_max_labels = int(slp_max_labels)
    p.slp_threshold = float(slp_threshold)
    return p


# ---------------------------------------------------------------- functions named like the ABI
def glp_nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(load_library().glp_nccl_unique_id(ctypes.cast(buf, ctypes.c_void_p)))
    return bytes(buf)


def glp_partition(n: int, nranks: int, row_offsets=None, edge_balanced: bool = False):
    import numpy as np
    out = np.zeros(nranks + 1, dtype=np.int64)
    off = None
    if row_offsets is not None:
        off = np.ascontiguousarray(row_offsets.cpu().numpy() if torch.is_tensor(row_offsets)
                                   else row_offsets, dtype=np.int64)
    _check(load_library().glp_partition(None if off is None else off.ctypes.data, int(n), int(nranks),
                                        int(bool(edge_balanced)), out.ctypes.data))
    return out.tolist()


def glp_graph_create(n_global: int, row_offsets: torch.Tensor, col_idx: torch.Tensor, *,
                     v_begin: int = 0, v_end: int | None = None, symmetric: bool = False,
                     rank: int = 0, nranks: int = 1, device: int | None = None,
                     nccl_unique_id: bytes | None = None, stream: torch.cuda.Stream | None = None,
                     validate: bool = True, local_group=None, host_arcs: bool = False, weights=None):
    """Create a device graph.  CUDA tensors are borrowed (keep them alive);
    CPU tensors are copied.  weights: optional per-arc integer weights in
    [1, 2^31) on the same device as col_idx (weighted LP).  Returns an opaque
    handle (ctypes.c_void_p)."""
    lib = load_library()
    if v_end is None:
        v_end = n_global
    on_device = row_offsets.is_cuda
    if col_idx.is_cuda != on_device:
        raise ValueError("row_offsets and col_idx must be on the same device")
    row_offsets = row_offsets.contiguous()
    col_idx = col_idx.contiguous()
    if row_offsets.dtype != torch.int64 or col_idx.dtype != torch.int32:
        raise TypeError("row_offsets must be int64 and col_idx int32")
    c = glp_csr()
    c.n_global = int(n_global)
    c.v_begin, c.v_end = int(v_begin), int(v_end)
    c.nnz_local = int(col_idx.numel())
    c.row_offsets = row_offsets.data_ptr()
    c.col_idx = col_idx.data_ptr() if col_idx.numel() else None
    c.on_device = int(on_device)
    c.symmetric = int(bool(symmetric))
    if weights is not None:
        if not torch.is_tensor(weights) or weights.dtype not in (torch.int32, torch.int64) \
                or weights.numel() != col_idx.numel() or weights.is_cuda != on_device:
            raise TypeError("weights: an int32/int64 tensor with one entry per arc, on col_idx's device")
        weights = weights.to(torch.int32).contiguous()  # uint32 bit pattern (values < 2^31)
        c.weights = weights.data_ptr() if weights.numel() else None
    d = None
    uid_buf = None
    if nranks > 1 or device is not None or stream is not None or local_group is not None:
        d = glp_dist()
        d.rank, d.nranks = int(rank), int(nranks)
        d.device = int(device if device is not None else
                       (row_offsets.device.index if on_device else torch.cuda.current_device()))
        if nccl_unique_id is not None:
            uid_buf = (ctypes.c_uint8 * 128).from_buffer_copy(nccl_unique_id)
            d.nccl_unique_id = ctypes.cast(uid_buf, ctypes.c_void_p)
        d.cuda_stream = stream.cuda_stream if stream is not None else None
        d.local_group = local_group
    if on_device and stream is None:
        # borrowed tensors are read on the library's own stream: they must be
        # complete (torch may still be producing them on its current stream)
        torch.cuda.current_stream(row_offsets.device).synchronize()
    h = ctypes.c_void_p()
    prm = make_params(validate=validate, host_arcs=host_arcs)
    st = lib.glp_graph_create(ctypes.byref(c), None if d is None else ctypes.byref(d), ctypes.byref(prm),
                              ctypes.byref(h))
    if st == 3 and torch.cuda.is_available():
        # GLP_ERR_OUT_OF_MEMORY: the library already trimmed its private pool
        # and retried; torch's caching allocator may still hold freed blocks,
        # so return them to the driver and try once more
        torch.cuda.empty_cache()
        st = lib.glp_graph_create(ctypes.byref(c), None if d is None else ctypes.byref(d), ctypes.byref(prm),
                                  ctypes.byref(h))
    _check(st)
    return h


def glp_run(handle, variant: int = CLASSIC, max_iters: int = 20, seeds=None, *, gamma: float = 0.0,
            frontier: int = -1, stop_on_2cycle: bool = True, profile: bool = False,
            dense_divisor: int = 0, debug_pred_cap: int = 0, llp_hist: int = 0, tail_cms: bool = False,
            cms_ht_slots: int = 0, cms_depth: int = 0, sparse_exchange: int = -1, slp_max_labels: int = 0,
            slp_threshold: float = 0.0) -> dict:
    import numpy as np
    lib = load_library()
    sd = None
    ns = 0
    if seeds is not None:
        sd = np.ascontiguousarray(seeds.cpu().numpy() if torch.is_tensor(seeds) else seeds, dtype=np.int32)
        ns = int(sd.size)
    info = glp_run_info()
    prm = make_params(gamma=gamma, frontier=frontier, stop_on_2cycle=stop_on_2cycle, profile=profile,
                      dense_divisor=dense_divisor, debug_pred_cap=debug_pred_cap, llp_hist=llp_hist,
                      tail_cms=tail_cms, cms_ht_slots=cms_ht_slots, cms_depth=cms_depth,
                      sparse_exchange=sparse_exchange, slp_max_labels=slp_max_labels, slp_threshold=slp_threshold)
    _check(lib.glp_run(handle, int(variant), int(max_iters), None if sd is None else sd.ctypes.data, ns,
                       ctypes.byref(prm), ctypes.byref(info)))
    return dict(iterations=info.iterations, stop_reason=info.stop_reason,
                changed_last=info.changed_last, arcs_processed=info.arcs_processed,
                elapsed_ms=info.elapsed_ms, kernel_launches=info.kernel_launches)


def glp_labels_get(handle, out: torch.Tensor) -> torch.Tensor:
    if out.dtype != torch.int32 or not out.is_contiguous():
        raise TypeError("out must be a contiguous int32 tensor")
    _check(load_library().glp_labels_get(handle, out.data_ptr() if out.numel() else None, out.numel(),
                                         int(out.is_cuda)))
    return out


def glp_iter_stats(handle) -> list:
    lib = load_library()
    n = ctypes.c_int32()
    _check(lib.glp_iter_stats(handle, None, 0, ctypes.byref(n)))
    arr = (glp_iter_stat * max(n.value, 1))()
    _check(lib.glp_iter_stats(handle, ctypes.cast(arr, ctypes.c_void_p), n.value, ctypes.byref(n)))
    return [dict(changed=s.changed, d2=s.d2, active_vertices=s.active_vertices, active_arcs=s.active_arcs,
                 dense=bool(s.dense), exchange=s.exchange, ms=s.ms, cms_rows=s.cms_rows, cms_rescans=s.cms_rescans,
                 cms_fallbacks=s.cms_fallbacks) for s in arr[:n.value]]


def glp_kernel_stats(handle) -> list:
    lib = load_library()
    n = ctypes.c_int32()
    _check(lib.glp_kernel_stats(handle, None, 0, ctypes.byref(n)))
    arr = (glp_kernel_stat * max(n.value, 1))()
    _check(lib.glp_kernel_stats(handle, ctypes.cast(arr, ctypes.c_void_p), n.value, ctypes.byref(n)))
    return [dict(name=s.name.decode(), launches=s.launches, ms=s.ms, bytes=s.bytes, arcs=s.arcs)
            for s in arr[:n.value]]


def glp_graph_info(handle) -> dict:
    import numpy as np
    out = np.zeros(16, dtype=np.int64)
    _check(load_library().glp_graph_info(handle, out.ctypes.data, 16))
    names = ["isolated", "low", "mid", "high", "huge"]
    bins = {nm: dict(vertices=int(out[2 + 2 * i]), arcs=int(out[3 + 2 * i])) for i, nm in enumerate(names)}
    return dict(n=int(out[0]), nnz=int(out[1]), bins=bins, max_degree=int(out[12]), low_chunks=int(out[13]))


def glp_slp_memory_get(handle, n_rows: int, K: int):
    """SLP candidates of this rank's rows: (labels [n_rows, K], counts [n_rows, K]) int32 CPU tensors."""
    lab = torch.empty((n_rows, K), dtype=torch.int32)
    cnt = torch.empty((n_rows, K), dtype=torch.int32)
    _check(load_library().glp_slp_memory_get(handle, lab.data_ptr() if lab.numel() else None,
                                             cnt.data_ptr() if cnt.numel() else None, lab.numel(), 0))
    return lab, cnt


def glp_local_group_create(nranks: int):
    """An in-process rank group (see glp.h): handle for glp_graph_create(local_group=...)."""
    h = ctypes.c_void_p()
    _check(load_library().glp_local_group_create(int(nranks), ctypes.byref(h)))
    return h


def glp_local_group_destroy(handle) -> None:
    if handle:
        _check(load_library().glp_local_group_destroy(handle))


def glp_graph_destroy(handle) -> None:
    if handle:
        _check(load_library().glp_graph_destroy(handle))


def glp_struct_sizes() -> list:
    import numpy as np
    out = np.zeros(6, dtype=np.int64)
    _check(load_library().glp_struct_sizes(out.ctypes.data, 6))
    return out.tolist()


def glp_version() -> str:
    return load_library().glp_version().decode()


# ---------------------------------------------------------------- convenience wrapper
@dataclass
class RunInfo:
    iterations: int
    stop_reason: int
    changed_last: int
    arcs_processed: int
    elapsed_ms: float
    kernel_launches: int

    @property
    def stop(self) -> str:
        return STOP_NAMES[self.stop_reason]


class Graph:
    """A device-resident CSR graph ready for label propagation.

    ``Graph(csr)`` accepts a ``glp_inputs.CSR`` (or n/row_offsets/col_idx).
    CUDA tensors are borrowed (the Graph keeps a reference); CPU tensors are
    copied to the device by the library.
    """

    def __init__(self, csr=None, *, n=None, row_offsets=None, col_idx=None, symmetric=None,
                 validate=True, weights=None, **dist):
        # symmetric: None = the CSR's own flag (glp_inputs.CSR.symmetric), else
        # False -- the frontier push is exact only on symmetric graphs, so it
        # is never assumed (the C ABI's zero default)
        if csr is not None:
            n, row_offsets, col_idx = csr.n, csr.row_offsets, csr.col_idx
            if symmetric is None:
                symmetric = bool(getattr(csr, "symmetric", False))
        symmetric = bool(symmetric) if symmetric is not None else False
        self.n = int(n)
        self._off = row_offsets
        self._col = col_idx
        if weights is not None and torch.is_tensor(weights) and weights.is_cuda:
            weights = weights.to(torch.int32).contiguous()
        self._w = weights
        self.device = row_offsets.device if row_offsets.is_cuda else torch.device("cuda", torch.cuda.current_device())
        self.handle = glp_graph_create(self.n, row_offsets, col_idx, symmetric=symmetric,
                                       validate=validate, weights=self._w, **dist)

    def run(self, variant="classic", max_iters: int = 20, seeds=None, **kw) -> RunInfo:
        v = VARIANTS[variant] if isinstance(variant, str) else int(variant)
        return RunInfo(**glp_run(self.handle, v, max_iters, seeds, **kw))

    def labels(self, device=None) -> torch.Tensor:
        dev = self.device if device is None else torch.device(device)
        out = torch.empty(self.n, dtype=torch.int32, device=dev)
        if dev.type == "cpu":
            out = out.pin_memory() if torch.cuda.is_available() else out
        return glp_labels_get(self.handle, out)

    def iter_stats(self):
        return glp_iter_stats(self.handle)

    def slp_memory(self, K: int = 5, n_rows=None):
        """Candidates of the last SLP run (K = the run's slp_max_labels)."""
        return glp_slp_memory_get(self.handle, self.n if n_rows is None else n_rows, K)

    def kernel_stats(self):
        return glp_kernel_stats(self.handle)

    def info(self):
        return glp_graph_info(self.handle)

    def close(self):
        if getattr(self, "handle", None):
            glp_graph_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
