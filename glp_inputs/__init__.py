"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

Holds generators and the CSR container only -- none of the label-propagation
arithmetic (that lives separately in ``oracle/`` and in the CUDA library).
"""
from .csr import CSR, from_edges, from_arrays, relabel, save_npz, load_npz  # noqa: F401
from . import graphs, rng  # noqa: F401
