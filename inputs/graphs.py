"""Seeded synthetic input graphs, shared by the oracle side and the CUDA side.

This module is an INPUT GENERATOR only: it holds none of the method's
arithmetic (no queue, no BFS). Both `oracle/` and the CUDA path consume the
CSR it builds; neither imports the other.

Recipes:

* Kronecker / R-MAT (BASELINE.json configs 1, 4, 5): Graph500 parameters
  A, B, C, D = .57, .19, .19, .05, M = edgefactor * 2**scale generated
  tuples, bit-by-bit quadrant choice, then a seeded bijective relabelling of
  the vertex ids (Graph500's random permutation). The paper's own social
  graphs (Table 1) are out of scope; Kronecker is the
  stand-in for "large fanout with a large standard deviation".
* 2-D grid, 4-neighbour, row-major ids (config 3): the road-map stand-in,
  "fanout of between 2 and 3, but deep" (Table 2).
* 4-ary heap tree (NEXT row 2): the paper's synthetic dataset, "10,485,760
  vertices, with a fanout of 4"; children of i are 4i+1..4i+4.

Random numbers are drawn with a counter-based generator (splitmix64
finaliser of (seed, counter)) in pure integer arithmetic, so the numpy
implementation here and the CUDA implementation in `inputs/csrc/tqgen.cu`
produce bit-identical edge lists for the same seed.

CSR convention: undirected graph stored symmetric, self
loops removed, duplicate edges removed, each row sorted ascending;
`row_ptr: int64[V+1]`, `col: int32[nnz]`.
"""
from __future__ import annotations

import dataclasses

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
GOLDEN = np.uint64(0x9E3779B97F4A7C15)

# Graph500 R-MAT quadrant probabilities as 32-bit integer thresholds
# (A, A+B, A+B+C) * 2**32, truncated. Integer thresholds make the numpy and
# CUDA generators agree bit for bit (no floating point in the choice).
RMAT_A, RMAT_B, RMAT_C = 0.57, 0.19, 0.19
T_A = int(RMAT_A * 2**32)
T_AB = int((RMAT_A + RMAT_B) * 2**32)
T_ABC = int((RMAT_A + RMAT_B + RMAT_C) * 2**32)


def _mix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    x = x.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        x ^= x >> np.uint64(30)
        x *= np.uint64(0xBF58476D1CE4E5B9)
        x ^= x >> np.uint64(27)
        x *= np.uint64(0x94D049BB133111EB)
        x ^= x >> np.uint64(31)
    return x


def hash2(seed: int, ctr: np.ndarray) -> np.ndarray:
    """Counter-based draw h(seed, ctr) = mix(mix(seed) + ctr * golden)."""
    s = _mix64(np.array([seed & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64))[0]
    with np.errstate(over="ignore"):
        return _mix64(s + np.asarray(ctr, dtype=np.uint64) * GOLDEN)


def perm_params(seed: int, scale: int):
    """Parameters of the seeded bijection on [0, 2**scale) (4 uint64)."""
    h = hash2(seed ^ 0x5EED5EED, np.arange(4, dtype=np.uint64))
    mask = (1 << scale) - 1
    m1 = int(h[0]) & mask | 1
    a1 = int(h[1]) & mask
    m2 = int(h[2]) & mask | 1
    a2 = int(h[3]) & mask
    return m1, a1, m2, a2


def permute_ids(x: np.ndarray, scale: int, seed: int) -> np.ndarray:
    """Seeded bijective relabelling of ids in [0, 2**scale).

    x -> x*m1 + a1 -> xorshift -> x*m2 + a2 -> xorshift, all mod 2**scale.
    Each step is invertible mod 2**scale (odd multiplier; x ^ (x >> s) with
    s >= 1), so the composition is a permutation.
    """
    mask = np.uint64((1 << scale) - 1)
    m1, a1, m2, a2 = (np.uint64(v) for v in perm_params(seed, scale))
    sh = np.uint64(max(1, scale // 2 + 1))
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = (x * m1 + a1) & mask
        x = x ^ (x >> sh)
        x = (x * m2 + a2) & mask
        x = x ^ (x >> sh)
    return x


def kronecker_edges(scale: int, edgefactor: int, seed: int):
    """Graph500-style R-MAT edge tuples (src, dst) as uint64 arrays.

    Edge i, level l draws r = h(seed, i*64 + l) >> 32 and picks quadrant
    A (0,0), B (0,1), C (1,0) or D (1,1); bit l of (src, dst) is set
    accordingly. Then both endpoints go through `permute_ids`.
    """
    if not (1 <= scale <= 31):
        raise ValueError("scale must be in [1, 31]")
    m = edgefactor << scale
    i = np.arange(m, dtype=np.uint64)
    src = np.zeros(m, dtype=np.uint64)
    dst = np.zeros(m, dtype=np.uint64)
    for lvl in range(scale):
        r = hash2(seed, i * np.uint64(64) + np.uint64(lvl)) >> np.uint64(32)
        q_b = (r >= T_A) & (r < T_AB)
        q_c = (r >= T_AB) & (r < T_ABC)
        q_d = r >= T_ABC
        bit = np.uint64(1) << np.uint64(lvl)
        src |= np.where(q_c | q_d, bit, np.uint64(0))
        dst |= np.where(q_b | q_d, bit, np.uint64(0))
    return permute_ids(src, scale, seed), permute_ids(dst, scale, seed)


def grid_edges(rows: int, cols: int):
    """4-neighbour grid, vertex (r, c) has id r*cols + c."""
    v = np.arange(rows * cols, dtype=np.uint64).reshape(rows, cols)
    right = (v[:, :-1].ravel(), v[:, 1:].ravel())
    down = (v[:-1, :].ravel(), v[1:, :].ravel())
    return np.concatenate([right[0], down[0]]), np.concatenate([right[1], down[1]])


def tree4_edges(n: int):
    """Heap-ordered 4-ary tree on n vertices: edges (parent(i), i), i >= 1."""
    i = np.arange(1, n, dtype=np.uint64)
    return (i - np.uint64(1)) // np.uint64(4), i


@dataclasses.dataclass
class CSR:
    """Symmetric, deduplicated, loop-free CSR (rows sorted ascending)."""

    n_vertices: int
    row_ptr: np.ndarray  # int64[V+1]
    col: np.ndarray  # int32[nnz]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)


def edges_to_csr(src, dst, n_vertices: int, name: str = "") -> CSR:
    """Symmetrise, drop self loops and duplicates, sort rows."""
    if n_vertices >= 2**31:
        raise ValueError("vertex ids must fit int32")
    src = np.asarray(src, dtype=np.uint64)
    dst = np.asarray(dst, dtype=np.uint64)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    nv = np.uint64(n_vertices)
    keys = np.concatenate([src * nv + dst, dst * nv + src])
    keys = np.unique(keys)
    row = (keys // nv).astype(np.int64)
    col = (keys % nv).astype(np.int32)
    counts = np.bincount(row, minlength=n_vertices).astype(np.int64)
    row_ptr = np.zeros(n_vertices + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSR(n_vertices, row_ptr, col, name)


def csr_from_adjacency(adj: np.ndarray, name: str = "") -> CSR:
    """CSR from a dense symmetric 0/1 adjacency matrix (tiny test graphs)."""
    n = adj.shape[0]
    u, v = np.nonzero(adj)
    return edges_to_csr(u, v, n, name)


def kronecker_csr(scale: int, edgefactor: int = 16, seed: int = 1) -> CSR:
    s, d = kronecker_edges(scale, edgefactor, seed)
    return edges_to_csr(s, d, 1 << scale, f"kron{scale}_ef{edgefactor}_s{seed}")


def grid_csr(rows: int, cols: int | None = None) -> CSR:
    cols = rows if cols is None else cols
    s, d = grid_edges(rows, cols)
    return edges_to_csr(s, d, rows * cols, f"grid{rows}x{cols}")


def tree4_csr(n: int) -> CSR:
    s, d = tree4_edges(n)
    return edges_to_csr(s, d, n, f"tree4_{n}")


def edge_weights(row_ptr, col, seed: int, wmax: int = 255) -> np.ndarray:
    """Seeded integer edge weights in [1, wmax], one per CSR entry, symmetric
    (w(u,v) = w(v,u)): h(seed, min(u,v) * 2^32 + max(u,v)) mod wmax + 1."""
    row_ptr = np.asarray(row_ptr)
    col = np.asarray(col, dtype=np.int64)
    rows = np.repeat(np.arange(row_ptr.size - 1, dtype=np.int64), np.diff(row_ptr))
    lo = np.minimum(rows, col).astype(np.uint64)
    hi = np.maximum(rows, col).astype(np.uint64)
    h = hash2(seed ^ 0x77E16475, (lo << np.uint64(32)) | hi)
    return (h % np.uint64(wmax) + np.uint64(1)).astype(np.int32)


def sample_roots(row_ptr: np.ndarray, n_roots: int, seed: int) -> np.ndarray:
    """Graph500-style roots: seeded uniform draws among vertices of degree >= 1.

    Draw j takes h(seed, j) mod V and walks forward (cyclically) to the next
    vertex with degree >= 1; duplicates are allowed to be skipped by redrawing.
    """
    row_ptr = np.asarray(row_ptr)
    deg = np.diff(row_ptr)
    nz = np.flatnonzero(deg > 0)
    if nz.size == 0:
        raise ValueError("graph has no edges")
    v = int(row_ptr.size - 1)
    roots: list[int] = []
    seen = set()
    ctr = 0
    while len(roots) < n_roots:
        h = int(hash2(seed, np.array([ctr], dtype=np.uint64))[0])
        ctr += 1
        cand = h % v
        k = np.searchsorted(nz, cand)
        r = int(nz[k % nz.size])
        if r in seen and len(seen) < nz.size:
            continue
        seen.add(r)
        roots.append(r)
    return np.array(roots, dtype=np.int32)
