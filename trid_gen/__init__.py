"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds none of the method's arithmetic: it only draws matrices.  The paper never says how
its test matrices were generated, so the recipe is ours:

* ``random_symmetric``: a_ij = a_ji = 2 u(seed, min(i,j), max(i,j)) - 1 in [-1, 1), where
  u = (splitmix64(seed*G ^ (r*n + c)) >> 11) * 2^-53 and G = 0x9E3779B97F4A7C15.  The same
  counter-based hash runs in numpy (uint64) and in torch (int64 two's complement, CPU or CUDA); the
  tests check the three are bit-identical, so no input file is ever copied.
* ``clustered_symmetric``: A = H_r ... H_1 diag(lam) H_1 ... H_r with r dense Householder
  reflectors drawn from the same hash (exact spectrum up to ~r*eps), lam either 32 tight clusters
  (config 4) or the closed-form 1-2-1 Toeplitz spectrum 2 - 2 cos(k pi / (n+1)).

Tensors are returned as row-major torch (n, n) float64; because they are symmetric the column-major
view used by the C-ABI is the same matrix.
"""
from __future__ import annotations

import math

import numpy as np
import torch

G = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
_MASK64 = (1 << 64) - 1


def _s64(x: int) -> int:
    """uint64 constant -> the int64 with the same bits."""
    x &= _MASK64
    return x - (1 << 64) if x >= (1 << 63) else x


# ---------------------------------------------------------------- numpy (uint64, defined wrap-around)
def _mix_np(key: np.ndarray) -> np.ndarray:
    z = key.astype(np.uint64) + np.uint64(G)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
    return z ^ (z >> np.uint64(31))


def uniform_np(seed: int, idx: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        key = np.uint64((seed * G) & _MASK64) ^ idx.astype(np.uint64)
        z = _mix_np(key)
    return (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def random_symmetric_np(n: int, seed: int) -> np.ndarray:
    i = np.arange(n, dtype=np.uint64)[:, None]
    j = np.arange(n, dtype=np.uint64)[None, :]
    r = np.minimum(i, j)
    c = np.maximum(i, j)
    with np.errstate(over="ignore"):
        return 2.0 * uniform_np(seed, r * np.uint64(n) + c) - 1.0


# ---------------------------------------------------------------- torch (int64 two's complement)
def _lsr(z: torch.Tensor, k: int) -> torch.Tensor:
    return (z >> k) & ((1 << (64 - k)) - 1)


def _mix_t(key: torch.Tensor) -> torch.Tensor:
    z = key + _s64(G)
    z = (z ^ _lsr(z, 30)) * _s64(M1)
    z = (z ^ _lsr(z, 27)) * _s64(M2)
    return z ^ _lsr(z, 31)


def uniform_t(seed: int, idx: torch.Tensor) -> torch.Tensor:
    z = _mix_t(idx ^ _s64(seed * G))
    return _lsr(z, 11).to(torch.float64) * (2.0 ** -53)


def random_symmetric(n: int, seed: int, device="cpu", out: torch.Tensor | None = None,
                     chunk: int = 2048) -> torch.Tensor:
    """Random symmetric n x n float64 matrix, entries uniform in [-1, 1)."""
    A = out if out is not None else torch.empty((n, n), dtype=torch.float64, device=device)
    dev = A.device
    cols = torch.arange(n, dtype=torch.int64, device=dev)
    for r0 in range(0, n, chunk):
        r1 = min(n, r0 + chunk)
        rows = torch.arange(r0, r1, dtype=torch.int64, device=dev)[:, None]
        lo = torch.minimum(rows, cols[None, :])
        hi = torch.maximum(rows, cols[None, :])
        A[r0:r1] = 2.0 * uniform_t(seed, lo * n + hi) - 1.0
    return A


def random_symmetric_rows(n: int, seed: int, rows, device="cpu", chunk: int = 2048) -> torch.Tensor:
    """Rows `rows` (global indices) of random_symmetric(n, seed), as a (len(rows), n) tensor.  For the
    symmetric matrix row c equals column c, so this is also the column-major storage of the columns
    `rows` (the multi-GPU block-cyclic local matrix)."""
    rows = torch.as_tensor(rows, dtype=torch.int64, device=device)
    A = torch.empty((rows.numel(), n), dtype=torch.float64, device=device)
    cols = torch.arange(n, dtype=torch.int64, device=device)
    for r0 in range(0, rows.numel(), chunk):
        r = rows[r0:r0 + chunk, None]
        lo = torch.minimum(r, cols[None, :])
        hi = torch.maximum(r, cols[None, :])
        A[r0:r0 + chunk] = 2.0 * uniform_t(seed, lo * n + hi) - 1.0
    return A


def block_cyclic_columns(n: int, colblock: int, nranks: int, rank: int) -> np.ndarray:
    """Global column indices stored by `rank` in the 1D block-cyclic layout (blocks of colblock columns,
    block B on rank B % nranks), in local order.  Pure index bookkeeping."""
    blocks = np.arange(rank, (n + colblock - 1) // colblock, nranks, dtype=np.int64)
    cols = (blocks[:, None] * colblock + np.arange(colblock, dtype=np.int64)[None, :]).ravel()
    return cols[cols < n]


def _vec_idx(t: int, n: int, device) -> torch.Tensor:
    return (1 << 62) + t * (1 << 32) + torch.arange(n, dtype=torch.int64, device=device)


def toeplitz121_eigs(n: int) -> np.ndarray:
    """Closed-form spectrum of tridiag(-1, 2, -1) (ascending)."""
    k = np.arange(1, n + 1, dtype=np.float64)
    return np.sort(2.0 - 2.0 * np.cos(k * math.pi / (n + 1)))


def cluster_eigs(n: int, seed: int, nclusters: int = 32) -> np.ndarray:
    """32 tight clusters c_j (1 + 1e-10 xi), c_j = -1 + 2 j / 31 (config 4)."""
    j = np.arange(n) * nclusters // max(n, 1)
    c = -1.0 + 2.0 * j / (nclusters - 1)
    xi = 2.0 * uniform_np(seed + 77, np.arange(n, dtype=np.uint64)) - 1.0
    return np.sort(c * (1.0 + 1e-10 * xi))


def clustered_symmetric(n: int, seed: int, kind: str = "clusters", r: int = 8, device="cpu"):
    """A = H_r ... H_1 diag(lam) H_1 ... H_r.  Returns (A, lam ascending as numpy)."""
    lam = cluster_eigs(n, seed) if kind == "clusters" else toeplitz121_eigs(n)
    A = torch.zeros((n, n), dtype=torch.float64, device=device)
    A.diagonal().copy_(torch.from_numpy(lam).to(device))
    for t in range(r):
        u = 2.0 * uniform_t(seed, _vec_idx(t, n, device)) - 1.0
        u = u / torch.linalg.vector_norm(u)
        y = A @ u
        uy = torch.dot(u, y)
        A.addr_(u, y, alpha=-2.0)
        A.addr_(y, u, alpha=-2.0)
        A.addr_(u, u, alpha=4.0 * float(uy))
    return A, lam


def toeplitz121(n: int) -> np.ndarray:
    return 2.0 * np.eye(n) - np.eye(n, k=1) - np.eye(n, k=-1)
