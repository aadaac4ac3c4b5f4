"""Edge list -> symmetric CSR (the graph layout of GLP's *Graph* structure).

PAPER.md [P:97 §3.1]: "The compressed sparse row (CSR) format is used to store
the graph structure."  Undirected inputs are stored symmetrised, as the paper's
Table 2 does for dblp/roadNet/youtube/aligraph/ljournal [P:255-264]; SURVEY
§8(c) reading 3: self-loops dropped, multi-edges deduplicated.

The CSR is a plain dataclass of two int64/int32 tensors; it carries no
label-propagation arithmetic.
"""
from __future__ import annotations

import hashlib
from dataclasses import dataclass

import numpy as np
import torch


@dataclass
class CSR:
    n: int
    row_offsets: torch.Tensor  # int64 [n+1]
    col_idx: torch.Tensor      # int32 [nnz]
    name: str = ""
    symmetric: bool = False    # builder-asserted u in N(v) <=> v in N(u)

    @property
    def nnz(self) -> int:
        return int(self.col_idx.numel())

    def to(self, device) -> "CSR":
        return CSR(self.n, self.row_offsets.to(device), self.col_idx.to(device), self.name, self.symmetric)

    def numpy(self):
        return (self.row_offsets.cpu().numpy().astype(np.int64, copy=False),
                self.col_idx.cpu().numpy().astype(np.int32, copy=False))

    def degrees(self) -> torch.Tensor:
        return self.row_offsets[1:] - self.row_offsets[:-1]

    def sha256(self) -> str:
        off, col = self.numpy()
        h = hashlib.sha256()
        h.update(np.int64(self.n).tobytes())
        h.update(np.ascontiguousarray(off).tobytes())
        h.update(np.ascontiguousarray(col).tobytes())
        return h.hexdigest()


def from_edges(n: int, src: torch.Tensor, dst: torch.Tensor, name: str = "",
               symmetrize: bool = True) -> CSR:
    """Build a CSR over vertices [0, n) from edge endpoints.

    symmetrize=True adds (v,u) for every (u,v); self-loops are removed and
    duplicate arcs merged (each remaining CSR entry is one vote [P:110]).
    Rows are sorted by column id.  Works on any torch device.
    """
    src = src.to(torch.int64).reshape(-1)
    dst = dst.to(torch.int64).reshape(-1)
    assert src.shape == dst.shape
    device = src.device
    keep = src != dst
    src, dst = src[keep], dst[keep]
    if symmetrize:
        src, dst = torch.cat([src, dst]), torch.cat([dst, src])
    if src.numel():
        assert int(src.min()) >= 0 and int(src.max()) < n
        assert int(dst.min()) >= 0 and int(dst.max()) < n
    key = torch.unique(src * n + dst)  # sorted, deduplicated
    del src, dst
    rows = torch.div(key, n, rounding_mode="floor")
    cols = (key - rows * n).to(torch.int32)
    counts = torch.bincount(rows, minlength=n) if n > 0 else torch.zeros(0, dtype=torch.int64, device=device)
    off = torch.zeros(n + 1, dtype=torch.int64, device=device)
    if n > 0:
        off[1:] = torch.cumsum(counts, 0)
    return CSR(n, off, cols.contiguous(), name, symmetrize)


def from_arrays(n: int, row_offsets, col_idx, name: str = "", symmetric: bool = False) -> CSR:
    """Wrap raw (possibly non-symmetric / unvalidated) arrays as a CSR; the
    caller states whether it is symmetric (default: not asserted)."""
    off = torch.as_tensor(np.asarray(row_offsets, dtype=np.int64))
    col = torch.as_tensor(np.asarray(col_idx, dtype=np.int32))
    return CSR(n, off, col, name, symmetric)


def relabel(csr: CSR, new_id: torch.Tensor) -> CSR:
    """Apply a vertex permutation (new_id[old] = new) and rebuild the CSR."""
    off = csr.row_offsets
    deg = off[1:] - off[:-1]
    rows = torch.repeat_interleave(torch.arange(csr.n, device=off.device), deg)
    src = new_id[rows]
    dst = new_id[csr.col_idx.to(torch.int64)]
    out = from_edges(csr.n, src, dst, csr.name, symmetrize=False)
    out.symmetric = csr.symmetric  # a permutation keeps (a)symmetry
    return out


def save_npz(csr: CSR, path: str) -> None:
    off, col = csr.numpy()
    np.savez(path, n=np.int64(csr.n), row_offsets=off, col_idx=col, name=np.str_(csr.name),
             symmetric=np.bool_(csr.symmetric))


def load_npz(path: str) -> CSR:
    z = np.load(path)
    return CSR(int(z["n"]), torch.from_numpy(z["row_offsets"]), torch.from_numpy(z["col_idx"]), str(z["name"]),
               bool(z["symmetric"]) if "symmetric" in z else False)
