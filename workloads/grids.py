"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the factorization method (no elimination,
no symbolic analysis, no front algebra).  It only builds the input matrices,
the fill-reducing order and right-hand sides, exactly as specified in
SURVEY.md Appendix B ("Exact specification of inputs and rules"), which
re-creates workloads shaped like the paper's test matrices
[PAPER.md L79-87, Table II: 3-D structural problems, 0.67-1.52 M unknowns].

Conventions:
  * matrices are returned as the LOWER triangle (row >= col, diagonal
    included) in 0-based CSC: ``colptr`` int64 (n+1), ``rowind`` int32,
    ``values`` float64, rows sorted ascending inside each column;
  * ``perm[k]`` = original index of the k-th pivot (new -> old).
"""
from __future__ import annotations

import sys
from dataclasses import dataclass

import numpy as np

__all__ = [
    "CSC", "nd_perm", "laplacian_1d", "laplacian_5pt", "laplacian_7pt",
    "stencil_9pt", "stencil_27pt", "elasticity_q1", "CONFIGS", "make_config",
    "rhs", "full_symmetric_dense", "random_spd_pattern",
]


@dataclass
class CSC:
    """Lower-triangular CSC of a symmetric matrix."""
    n: int
    colptr: np.ndarray  # int64, n+1
    rowind: np.ndarray  # int32, nnz
    values: np.ndarray  # float64, nnz

    @property
    def nnz(self) -> int:
        return int(self.colptr[-1])


# --------------------------------------------------------------------------
# Geometric nested dissection ("Geometric nested dissection")
# --------------------------------------------------------------------------
def nd_perm(nx: int, ny: int = 1, nz: int = 1, dof: int = 1) -> np.ndarray:
    """perm[k] = old id of the k-th emitted node; old id v = (z*NY + y)*NX + x.

    nd(box): if an extent <= 0 return; split the axis with the strictly largest
    extent (ties x before y before z); if that extent is 1 emit the node;
    mid = lo + extent//2; recurse on [lo, mid), then [mid+1, hi); then emit the
    plane at mid (axis x: for z, for y; axis y: for z, for x; axis z: for y, for x;
    the second-named coordinate varies fastest).  With ``dof`` > 1 every node v
    expands to dofs dof*v + c, c = 0..dof-1.
    """
    out: list[np.ndarray] = []
    sys.setrecursionlimit(max(10000, sys.getrecursionlimit()))

    def emit_plane(axis, mid, x0, x1, y0, y1, z0, z1):
        if axis == 0:   # for z, for y (y fastest)
            zz, yy = np.meshgrid(np.arange(z0, z1), np.arange(y0, y1), indexing="ij")
            v = (zz * ny + yy) * nx + mid
        elif axis == 1:  # for z, for x
            zz, xx = np.meshgrid(np.arange(z0, z1), np.arange(x0, x1), indexing="ij")
            v = (zz * ny + mid) * nx + xx
        else:            # for y, for x
            yy, xx = np.meshgrid(np.arange(y0, y1), np.arange(x0, x1), indexing="ij")
            v = (mid * ny + yy) * nx + xx
        out.append(v.reshape(-1).astype(np.int64))

    def nd(x0, x1, y0, y1, z0, z1):
        ex, ey, ez = x1 - x0, y1 - y0, z1 - z0
        if ex <= 0 or ey <= 0 or ez <= 0:
            return
        if ex >= ey and ex >= ez:
            axis, e = 0, ex
        elif ey >= ez:
            axis, e = 1, ey
        else:
            axis, e = 2, ez
        if e == 1:
            out.append(np.array([(z0 * ny + y0) * nx + x0], dtype=np.int64))
            return
        if axis == 0:
            mid = x0 + ex // 2
            nd(x0, mid, y0, y1, z0, z1)
            nd(mid + 1, x1, y0, y1, z0, z1)
        elif axis == 1:
            mid = y0 + ey // 2
            nd(x0, x1, y0, mid, z0, z1)
            nd(x0, x1, mid + 1, y1, z0, z1)
        else:
            mid = z0 + ez // 2
            nd(x0, x1, y0, y1, z0, mid)
            nd(x0, x1, y0, y1, mid + 1, z1)
        emit_plane(axis, mid, x0, x1, y0, y1, z0, z1)

    nd(0, nx, 0, ny, 0, nz)
    p = np.concatenate(out)
    assert p.size == nx * ny * nz
    if dof > 1:
        p = (dof * p[:, None] + np.arange(dof)[None, :]).reshape(-1)
    return p.astype(np.int32)


# --------------------------------------------------------------------------
# Stencil matrices ("Matrices"; reading C13)
# --------------------------------------------------------------------------
def _stencil(nx: int, ny: int, nz: int, offsets: list[tuple[int, int, int, float]]) -> CSC:
    """Lower CSC of a constant-coefficient stencil on an nx*ny*nz grid (Dirichlet:
    neighbours outside the grid are dropped).  ``offsets`` lists (dx,dy,dz,coef),
    only those whose linear delta is >= 0 (lower triangle incl. diagonal) are used."""
    n = nx * ny * nz
    lin = [(dz * ny * nx + dy * nx + dx, dx, dy, dz, c) for dx, dy, dz, c in offsets]
    lin = sorted([t for t in lin if t[0] >= 0])
    v = np.arange(n, dtype=np.int64)
    x = v % nx
    y = (v // nx) % ny
    z = v // (nx * ny)
    cols, rows, vals = [], [], []
    for delta, dx, dy, dz, c in lin:
        ok = (x + dx >= 0) & (x + dx < nx) & (y + dy >= 0) & (y + dy < ny) & (z + dz >= 0) & (z + dz < nz)
        cv = v[ok]
        cols.append(cv)
        rows.append(cv + delta)
        vals.append(np.full(cv.size, c, dtype=np.float64))
    cols = np.concatenate(cols)
    rows = np.concatenate(rows)
    vals = np.concatenate(vals)
    order = np.argsort(cols, kind="stable")  # offsets were emitted in ascending delta
    cols, rows, vals = cols[order], rows[order], vals[order]
    colptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(cols, minlength=n), out=colptr[1:])
    return CSC(n, colptr, rows.astype(np.int32), vals)


def laplacian_1d(n: int) -> CSC:
    """tridiag(-1, 2, -1) ("1D chain")."""
    return _stencil(n, 1, 1, [(0, 0, 0, 2.0), (1, 0, 0, -1.0)])


def laplacian_5pt(nx: int, ny: int | None = None) -> CSC:
    """K (x) I + I (x) K, diagonal 4."""
    ny = nx if ny is None else ny
    return _stencil(nx, ny, 1, [(0, 0, 0, 4.0), (1, 0, 0, -1.0), (0, 1, 0, -1.0)])


def laplacian_7pt(nx: int, ny: int | None = None, nz: int | None = None) -> CSC:
    """K(x)I(x)I + I(x)K(x)I + I(x)I(x)K, diagonal 6."""
    ny = nx if ny is None else ny
    nz = nx if nz is None else nz
    return _stencil(nx, ny, nz, [(0, 0, 0, 6.0), (1, 0, 0, -1.0), (0, 1, 0, -1.0), (0, 0, 1, -1.0)])


def stencil_9pt(nx: int, ny: int | None = None) -> CSC:
    """9I - T(x)T with T = tridiag(1,1,1): diagonal 8, all 8 neighbours -1."""
    ny = nx if ny is None else ny
    offs = [(dx, dy, 0, 8.0 if (dx, dy) == (0, 0) else -1.0) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    return _stencil(nx, ny, 1, offs)


def stencil_27pt(nx: int, ny: int | None = None, nz: int | None = None) -> CSC:
    """27I - T(x)T(x)T: diagonal 26, all 26 neighbours -1."""
    ny = nx if ny is None else ny
    nz = nx if nz is None else nz
    offs = [(dx, dy, dz, 26.0 if (dx, dy, dz) == (0, 0, 0) else -1.0)
            for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    return _stencil(nx, ny, nz, offs)


def _q1_element_matrix() -> np.ndarray:
    """36 * K_e for a unit trilinear hexahedron, lambda = mu = 1, 2x2x2 Gauss
    (integer entries in [-8, 20], six rigid-body modes).
    Local node a = (x,y,z) in {0,1}^3 ordered x fastest; dof 3a + c."""
    g = 1.0 / np.sqrt(3.0)
    corners = [(x, y, z) for z in (0, 1) for y in (0, 1) for x in (0, 1)]
    D = np.full((6, 6), 0.0)
    D[:3, :3] = 1.0                         # lambda
    D += np.diag([2.0, 2.0, 2.0, 1.0, 1.0, 1.0])  # 2 mu, mu
    K = np.zeros((24, 24))
    for xi in (-g, g):
        for eta in (-g, g):
            for zeta in (-g, g):
                B = np.zeros((6, 24))
                for a, (x, y, z) in enumerate(corners):
                    sx, sy, sz = 2 * x - 1, 2 * y - 1, 2 * z - 1
                    dx = 2 * sx * (1 + sy * eta) * (1 + sz * zeta) / 8
                    dy = 2 * sy * (1 + sx * xi) * (1 + sz * zeta) / 8
                    dz = 2 * sz * (1 + sx * xi) * (1 + sy * eta) / 8
                    B[0, 3 * a], B[1, 3 * a + 1], B[2, 3 * a + 2] = dx, dy, dz
                    B[3, 3 * a], B[3, 3 * a + 1] = dy, dx
                    B[4, 3 * a + 1], B[4, 3 * a + 2] = dz, dy
                    B[5, 3 * a], B[5, 3 * a + 2] = dz, dx
                K += B.T @ D @ B / 8.0
    Ki = np.rint(36.0 * K)
    assert np.abs(Ki - 36.0 * K).max() < 1e-9
    return Ki


def elasticity_q1(N: int) -> CSC:
    """Q1 linear elasticity, 3 dof/node, clamped on all faces (SURVEY.md Appendix B,
    "Elasticity assembly"): node lattice (N+2)^3, (N+1)^3 unit elements, boundary
    nodes removed -> N^3 free nodes, dof 3v+c with v = (z*N+y)*N+x over free nodes.
    The full 3x3 block of every node pair sharing an element is stored (explicit
    zeros kept), giving the 27-point node pattern."""
    Ke = _q1_element_matrix()
    corners = np.array([(x, y, z) for z in (0, 1) for y in (0, 1) for x in (0, 1)], dtype=np.int64)
    e = np.arange(N + 1, dtype=np.int64)
    ez, ey, ex = np.meshgrid(e, e, e, indexing="ij")
    ex, ey, ez = ex.ravel(), ey.ravel(), ez.ravel()
    # free-node id of every element corner (-1 if on the clamped boundary)
    gid = np.empty((ex.size, 8), dtype=np.int64)
    for a, (cx, cy, cz) in enumerate(corners):
        X, Y, Z = ex + cx, ey + cy, ez + cz
        free = (X >= 1) & (X <= N) & (Y >= 1) & (Y <= N) & (Z >= 1) & (Z <= N)
        gid[:, a] = np.where(free, ((Z - 1) * N + (Y - 1)) * N + (X - 1), -1)
    n = 3 * N ** 3
    rows_l, cols_l, vals_l = [], [], []
    for a in range(8):
        for b in range(8):
            ok = (gid[:, a] >= 0) & (gid[:, b] >= 0)
            ga, gb = gid[ok, a], gid[ok, b]
            for ca in range(3):
                for cb in range(3):
                    r = 3 * ga + ca
                    c = 3 * gb + cb
                    low = r >= c
                    rows_l.append(r[low])
                    cols_l.append(c[low])
                    vals_l.append(np.full(int(low.sum()), Ke[3 * a + ca, 3 * b + cb]))
    r = np.concatenate(rows_l)
    c = np.concatenate(cols_l)
    v = np.concatenate(vals_l)
    key = c * n + r
    order = np.argsort(key, kind="stable")
    key, v = key[order], v[order]
    uniq, start = np.unique(key, return_index=True)
    sums = np.add.reduceat(v, start)  # element contributions are small integers: exact
    cols = uniq // n
    rows = uniq % n
    colptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(cols, minlength=n), out=colptr[1:])
    return CSC(n, colptr, rows.astype(np.int32), sums.astype(np.float64))


# --------------------------------------------------------------------------
# BASELINE.json configs (SURVEY.md §8(d) "Algorithmic work per config")
# --------------------------------------------------------------------------
CONFIGS = {
    "c1": dict(desc="2D 5-point Laplacian 32x32 grid (n=1024), nested dissection", kind="5pt", N=32),
    "c2": dict(desc="2D 9-point Laplacian 1000x1000 grid (n=1M), nested dissection", kind="9pt", N=1000),
    "c3": dict(desc="3D 7-point Laplacian 64^3 (n=262k), nested dissection", kind="7pt", N=64),
    "c4": dict(desc="3D linear elasticity 3 dof/node 50^3 grid (n=375k), nested dissection", kind="elast", N=50),
    "c5": dict(desc="3D 27-point stencil 100^3 (n=1M), nested dissection", kind="27pt", N=100),
}


def make_config(kind: str, N: int) -> tuple[CSC, np.ndarray]:
    """(matrix, ND perm) for a grid family at size N."""
    if kind == "1d":
        return laplacian_1d(N), np.arange(N, dtype=np.int32)
    if kind == "5pt":
        return laplacian_5pt(N), nd_perm(N, N)
    if kind == "9pt":
        return stencil_9pt(N), nd_perm(N, N)
    if kind == "7pt":
        return laplacian_7pt(N), nd_perm(N, N, N)
    if kind == "27pt":
        return stencil_27pt(N), nd_perm(N, N, N)
    if kind == "elast":
        return elasticity_q1(N), nd_perm(N, N, N, dof=3)
    raise ValueError(kind)


def rhs(n: int, seed: int = 0) -> np.ndarray:
    """x* ~ U(-1, 1) from numpy PCG64(seed) (SURVEY.md §8(d) "Seeds")."""
    return np.random.Generator(np.random.PCG64(seed)).uniform(-1.0, 1.0, n)


def full_symmetric_dense(A: CSC) -> np.ndarray:
    """Dense symmetric matrix from the lower CSC (duplicates summed)."""
    M = np.zeros((A.n, A.n))
    cols = np.repeat(np.arange(A.n), np.diff(A.colptr))
    r = A.rowind.astype(np.int64)
    keep = r >= cols
    np.add.at(M, (r[keep], cols[keep]), A.values[keep])
    d = np.diag(np.diag(M))
    return M + M.T - d


def random_spd_pattern(n: int, density: float, seed: int, dup: float = 0.0, upper: float = 0.0) -> CSC:
    """Random sparse SPD matrix (diagonally dominant), lower CSC, possibly with
    duplicate entries (``dup`` fraction, FEM style) and stray upper-triangle
    entries (``upper`` fraction; the boundary ignores them)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    m = int(density * n * (n - 1) / 2)
    r = rng.integers(0, n, m)
    c = rng.integers(0, n, m)
    keep = r != c
    r, c = np.maximum(r[keep], c[keep]), np.minimum(r[keep], c[keep])
    v = -rng.uniform(0.1, 1.0, r.size)
    nd = int(dup * r.size)
    if nd:
        idx = rng.integers(0, r.size, nd)
        r = np.concatenate([r, r[idx]]); c = np.concatenate([c, c[idx]])
        v = np.concatenate([v, -rng.uniform(0.1, 1.0, nd)])
    rowsum = np.bincount(r, weights=-v, minlength=n) + np.bincount(c, weights=-v, minlength=n)
    diag_r = np.arange(n)
    rr = np.concatenate([r, diag_r]); cc = np.concatenate([c, diag_r])
    vv = np.concatenate([v, rowsum + 1.0 + rng.uniform(0, 1, n)])
    nu = int(upper * r.size)
    if nu:
        idx = rng.integers(0, r.size, nu)
        rr = np.concatenate([rr, c[idx]]); cc = np.concatenate([cc, r[idx]])
        vv = np.concatenate([vv, rng.uniform(-5, 5, nu)])  # ignored by the lower-only convention
    order = rng.permutation(rr.size)  # unsorted rows inside columns are allowed
    rr, cc, vv = rr[order], cc[order], vv[order]
    order = np.argsort(cc, kind="stable")
    rr, cc, vv = rr[order], cc[order], vv[order]
    colptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(cc, minlength=n), out=colptr[1:])
    return CSC(n, colptr, rr.astype(np.int32), vv)


def manufactured(n: int, Lp: np.ndarray, Li: np.ndarray, perm: np.ndarray, seed: int = 1234):
    """Manufactured SPD matrix with an exactly known integer factor
    (SURVEY.md Sec. 8(c) "Manufactured exact factor"): L0 = +1 on the given
    off-diagonal structure (final labels, struct(L_j) ascending with j first),
    diagonal 2^p_j with p_j in {1,2,3} drawn from PCG64(seed); A = L0 L0^T,
    returned as the lower CSC in ORIGINAL labels (A_orig[perm[i], perm[j]] =
    A[i, j]).  Returns (CSC, L0 values aligned with Li)."""
    import scipy.sparse as sp
    rng = np.random.Generator(np.random.PCG64(seed))
    p = rng.integers(1, 4, n)
    Lx = np.ones(Li.size)
    Lx[Lp[:-1]] = 2.0 ** p                       # first entry of each column = diagonal
    L0 = sp.csc_matrix((Lx, Li, Lp), shape=(n, n))
    A = (L0 @ L0.T).tocoo()
    perm = np.asarray(perm, dtype=np.int64)
    r, c = perm[A.row], perm[A.col]
    keep = r >= c
    r, c, v = r[keep], c[keep], A.data[keep]
    order = np.lexsort((r, c))
    r, c, v = r[order], c[order], v[order]
    colptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(c, minlength=n), out=colptr[1:])
    return CSC(n, colptr, r.astype(np.int32), v), Lx
