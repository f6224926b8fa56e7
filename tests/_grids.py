"""Test helpers: build a grid matrix + ND perm by family and dims."""
from workloads import grids as G


def grid(kind, dims):
    nx, ny, nz = dims
    if kind == "5pt":
        return G.laplacian_5pt(nx, ny), G.nd_perm(nx, ny)
    if kind == "9pt":
        return G.stencil_9pt(nx, ny), G.nd_perm(nx, ny)
    if kind == "7pt":
        return G.laplacian_7pt(nx, ny, nz), G.nd_perm(nx, ny, nz)
    if kind == "27pt":
        return G.stencil_27pt(nx, ny, nz), G.nd_perm(nx, ny, nz)
    if kind == "elast":
        assert nx == ny == nz
        return G.elasticity_q1(nx), G.nd_perm(nx, nx, nx, dof=3)
    raise ValueError(kind)


def dense_from_rows(rows):
    """Lower CSC of a small dense symmetric matrix given as nested lists."""
    import numpy as np
    M = np.array(rows, dtype=float)
    n = M.shape[0]
    cols, rs, vs = [], [], []
    colptr = [0]
    for j in range(n):
        for i in range(j, n):
            if M[i, j] != 0 or i == j:
                rs.append(i); vs.append(M[i, j])
        colptr.append(len(rs))
    return G.CSC(n, np.array(colptr, dtype=np.int64), np.array(rs, dtype=np.int32), np.array(vs))
