"""Data-graph generators producing canonical undirected CSR.

Canonical CSR: ``row_ptr`` u64[n+1], ``col`` u32[nnz],
symmetric (every undirected edge {u,v} is stored as (u,v) and (v,u), the
undirected→directed conversion of PAPER.md:207-209, §2.1 Def. 1), each row
strictly ascending, no self loops, no duplicates.  Isolated vertices are kept.

Generators are deterministic functions of their seed:

* ``er_graph(n, m, seed)`` — Erdős–Rényi G(n, m): uniform unordered pairs from
  a numpy PCG64 stream, self loops and repeats rejected, until m distinct edges.
* ``rmat_graph(scale, ef, a, b, c, seed)`` — R-MAT: ef·2^scale samples; for each
  sample and each bit a quadrant is chosen from a splitmix64 counter-based
  uniform (keyed by seed, sample, bit); vertex ids are then relabelled by a
  seeded random permutation (id order creates imbalance),
  self loops dropped, symmetrised, deduplicated, rows sorted.
"""
from __future__ import annotations

from dataclasses import dataclass
import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


@dataclass(frozen=True)
class CSRGraph:
    n: int
    row_ptr: np.ndarray  # uint64[n+1]
    col: np.ndarray      # uint32[nnz]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def m(self) -> int:
        """Undirected edge count."""
        return self.nnz // 2

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr).astype(np.int64)

    def neighbors(self, v: int) -> np.ndarray:
        return self.col[int(self.row_ptr[v]):int(self.row_ptr[v + 1])]

    def edge_list(self) -> np.ndarray:
        """Undirected edges (u < v) as an (m, 2) int64 array."""
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.row_ptr).astype(np.int64))
        dst = self.col.astype(np.int64)
        keep = src < dst
        return np.stack([src[keep], dst[keep]], axis=1)


def canonical_csr(n: int, src, dst, name: str = "") -> CSRGraph:
    """Symmetrise, drop self loops, dedupe and sort an edge list into CSR."""
    src = np.asarray(src, dtype=np.uint64)
    dst = np.asarray(dst, dtype=np.uint64)
    if src.size:
        if int(src.max()) >= n or int(dst.max()) >= n:
            raise ValueError("edge endpoint out of range")
    keep = src != dst
    src, dst = src[keep], dst[keep]
    keys = np.concatenate([(src << np.uint64(32)) | dst, (dst << np.uint64(32)) | src])
    keys = np.unique(keys)  # sorted ascending: by row, then by column
    rows = (keys >> np.uint64(32)).astype(np.int64)
    col = (keys & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    counts = np.bincount(rows, minlength=n).astype(np.uint64)
    row_ptr = np.zeros(n + 1, dtype=np.uint64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSRGraph(n=n, row_ptr=row_ptr, col=col, name=name)


def graph_from_edges(n: int, edges, name: str = "") -> CSRGraph:
    e = np.asarray(list(edges), dtype=np.int64).reshape(-1, 2)
    return canonical_csr(n, e[:, 0], e[:, 1], name=name)


# --------------------------------------------------------------------------- ER
def er_graph(n: int, m: int, seed: int = 1) -> CSRGraph:
    """G(n, m): uniform unordered pairs, rejecting loops and duplicates."""
    if m > n * (n - 1) // 2:
        raise ValueError("too many edges")
    rng = np.random.Generator(np.random.PCG64(seed))
    seen: dict[int, None] = {}
    while len(seen) < m:
        need = m - len(seen)
        batch = max(2 * need, 64)
        u = rng.integers(0, n, size=batch, dtype=np.int64)
        v = rng.integers(0, n, size=batch, dtype=np.int64)
        for a, b in zip(u.tolist(), v.tolist()):
            if a == b:
                continue
            key = (min(a, b) << 32) | max(a, b)
            if key in seen:
                continue
            seen[key] = None
            if len(seen) == m:
                break
    keys = np.fromiter(seen.keys(), dtype=np.int64, count=m)
    return canonical_csr(n, keys >> 32, keys & 0xFFFFFFFF, name=f"er_n{n}_m{m}_s{seed}")


# ------------------------------------------------------------------------ R-MAT
def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser over uint64 (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def rmat_edges(scale: int, ef: int, a: float, b: float, c: float, seed: int = 1,
               block: int = 1 << 22):
    """Raw R-MAT samples (src, dst) before relabelling, as uint64 arrays."""
    nsamp = ef << scale
    t1, t2, t3 = a, a + b, a + b + c
    src = np.zeros(nsamp, dtype=np.uint64)
    dst = np.zeros(nsamp, dtype=np.uint64)
    key = splitmix64(np.array([seed], dtype=np.uint64))[0]
    inv = 1.0 / float(1 << 53)
    for s0 in range(0, nsamp, block):
        s1 = min(nsamp, s0 + block)
        ids = np.arange(s0, s1, dtype=np.uint64)
        su = np.zeros(s1 - s0, dtype=np.uint64)
        du = np.zeros(s1 - s0, dtype=np.uint64)
        with np.errstate(over="ignore"):
            base = ids * np.uint64(scale)
            for bit in range(scale):
                r = splitmix64(key ^ (base + np.uint64(bit)))
                u = (r >> np.uint64(11)).astype(np.float64) * inv
                sbit = (u >= t2).astype(np.uint64)                       # quadrants c, d
                dbit = (((u >= t1) & (u < t2)) | (u >= t3)).astype(np.uint64)  # quadrants b, d
                su = (su << np.uint64(1)) | sbit
                du = (du << np.uint64(1)) | dbit
        src[s0:s1] = su
        dst[s0:s1] = du
    return src, dst


def rmat_graph(scale: int, ef: int, a: float = 0.57, b: float = 0.19, c: float = 0.19,
               seed: int = 1) -> CSRGraph:
    n = 1 << scale
    src, dst = rmat_edges(scale, ef, a, b, c, seed)
    perm = np.random.Generator(np.random.PCG64(seed ^ 0xA5A5)).permutation(n).astype(np.uint64)
    src = perm[src.astype(np.int64)]
    dst = perm[dst.astype(np.int64)]
    return canonical_csr(n, src, dst, name=f"rmat_s{scale}_ef{ef}_a{a}_b{b}_c{c}_seed{seed}")


# ------------------------------------------------------------ structured graphs
def complete_graph(n: int) -> CSRGraph:
    return graph_from_edges(n, [(i, j) for i in range(n) for j in range(i + 1, n)], name=f"K{n}")


def cycle_graph(n: int) -> CSRGraph:
    return graph_from_edges(n, [(i, (i + 1) % n) for i in range(n)], name=f"C{n}")


def path_graph(n: int) -> CSRGraph:
    return graph_from_edges(n, [(i, i + 1) for i in range(n - 1)], name=f"P{n}")


def star_graph(s: int) -> CSRGraph:
    return graph_from_edges(s + 1, [(0, i) for i in range(1, s + 1)], name=f"K1_{s}")


def complete_bipartite_graph(a: int, b: int) -> CSRGraph:
    return graph_from_edges(a + b, [(i, a + j) for i in range(a) for j in range(b)], name=f"K{a}_{b}")


def grid_graph(r: int, c: int, keep: float = 1.0, seed: int = 1) -> CSRGraph:
    edges = []
    for i in range(r):
        for j in range(c):
            v = i * c + j
            if j + 1 < c:
                edges.append((v, v + 1))
            if i + 1 < r:
                edges.append((v, v + c))
    if keep < 1.0:
        rng = np.random.Generator(np.random.PCG64(seed))
        mask = rng.random(len(edges)) < keep
        edges = [e for e, k in zip(edges, mask) if k]
    return graph_from_edges(r * c, edges, name=f"grid{r}x{c}_keep{keep}")


def petersen_graph() -> CSRGraph:
    outer = [(i, (i + 1) % 5) for i in range(5)]
    spokes = [(i, i + 5) for i in range(5)]
    inner = [(5 + i, 5 + (i + 2) % 5) for i in range(5)]
    return graph_from_edges(10, outer + spokes + inner, name="petersen")


def hypercube_graph(d: int) -> CSRGraph:
    n = 1 << d
    return graph_from_edges(n, [(v, v ^ (1 << b)) for v in range(n) for b in range(d) if v < v ^ (1 << b)],
                            name=f"Q{d}")


# ----------------------------------------------- R-MAT, torch (same bytes, faster)
def _i64(x: int) -> int:
    """uint64 constant as the int64 with the same bit pattern."""
    return x - (1 << 64) if x >= 1 << 63 else x


def _srl(x, s: int):
    """Logical right shift of int64 tensors viewed as uint64."""
    import torch
    return (x >> s) & torch.tensor((1 << (64 - s)) - 1, dtype=torch.int64, device=x.device)


def _splitmix64_t(x):
    z = x + _i64(0x9E3779B97F4A7C15)
    z = (z ^ _srl(z, 30)) * _i64(0xBF58476D1CE4E5B9)
    z = (z ^ _srl(z, 27)) * _i64(0x94D049BB133111EB)
    return z ^ _srl(z, 31)


def rmat_graph_torch(scale: int, ef: int, a: float = 0.57, b: float = 0.19, c: float = 0.19,
                     seed: int = 1, device: str = "cpu", block: int = 1 << 24) -> CSRGraph:
    """``rmat_graph`` computed with torch int64 ops (wrapping, logical shifts) —
    byte-identical output (tests/test_oracle.py checks it), but fast enough on a
    GPU for the scale-20/22 configs.  The relabelling permutation is numpy's."""
    import torch
    n = 1 << scale
    nsamp = ef << scale
    t1, t2, t3 = a, a + b, a + b + c
    key = int(splitmix64(np.array([seed], dtype=np.uint64))[0])
    key_t = torch.tensor(_i64(key), dtype=torch.int64, device=device)
    perm_np = np.random.Generator(np.random.PCG64(seed ^ 0xA5A5)).permutation(n).astype(np.int64)
    perm = torch.from_numpy(perm_np).to(device)
    inv = 1.0 / float(1 << 53)
    keys = []
    for s0 in range(0, nsamp, block):
        s1 = min(nsamp, s0 + block)
        base = torch.arange(s0, s1, dtype=torch.int64, device=device) * scale
        su = torch.zeros(s1 - s0, dtype=torch.int64, device=device)
        du = torch.zeros_like(su)
        for bit in range(scale):
            r = _splitmix64_t(key_t ^ (base + bit))
            u = _srl(r, 11).to(torch.float64) * inv
            sbit = (u >= t2).to(torch.int64)
            dbit = (((u >= t1) & (u < t2)) | (u >= t3)).to(torch.int64)
            su = (su << 1) | sbit
            du = (du << 1) | dbit
        src, dst = perm[su], perm[du]
        keep = src != dst
        src, dst = src[keep], dst[keep]
        keys.append((src << 32) | dst)
        keys.append((dst << 32) | src)
    k = torch.unique(torch.cat(keys)) if keys else torch.zeros(0, dtype=torch.int64, device=device)
    rows = k >> 32
    col = (k & 0xFFFFFFFF).to(torch.int64)
    counts = torch.bincount(rows, minlength=n)
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    torch.cumsum(counts, 0, out=row_ptr[1:])
    return CSRGraph(n=n, row_ptr=row_ptr.cpu().numpy().astype(np.uint64),
                    col=col.cpu().numpy().astype(np.uint32),
                    name=f"rmat_s{scale}_ef{ef}_a{a}_b{b}_c{c}_seed{seed}")
