"""CPU pin of the premise behind the DIA-27 reading of the SpMV
(HPCCG_OPT_SPMV_FORMAT = 1), checked on the ORACLE's own
generator (oracle/, independent of the CUDA path): in the HPCCG 27-point
matrix (BJ:north_star: diag 27, -1 per existing neighbour of the 3x3x3
stencil, truncated at the domain boundary) every stored entry of row g is
nonzero and sits at column g + sz*nx*ny + sy*nx + sx for exactly the
in-domain neighbours (sx, sy, sz) in {-1, 0, 1}^3 -- so a column is a function
of (row, stencil slot, value != 0), and a kernel may form it instead of
loading it.  Brute force over every row of small grids, z-slabs included."""
import numpy as np
import pytest

import oracle


@pytest.mark.parametrize("dims,rank,nranks", [((5, 4, 3), 0, 1), ((1, 1, 1), 0, 1), ((7, 2, 1), 0, 1),
                                              ((6, 5, 2), 1, 3), ((4, 3, 3), 2, 3), ((2, 9, 2), 0, 2)])
def test_columns_are_stencil_offsets_of_nonzeros(dims, rank, nranks):
    nx, ny, nz = dims
    prob = oracle.generate(nx, ny, nz, rank, nranks)
    n, plane, nzg = nx * ny * nz, nx * ny, nz * nranks
    rp = prob.row_ptr
    for i in range(n):
        g = rank * n + i
        gz, rem = divmod(g, plane)
        iy, ix = divmod(rem, nx)
        expect = []
        for sz in (-1, 0, 1):
            for sy in (-1, 0, 1):
                for sx in (-1, 0, 1):
                    if 0 <= ix + sx < nx and 0 <= iy + sy < ny and 0 <= gz + sz < nzg:
                        expect.append((g + sz * plane + sy * nx + sx,
                                       27.0 if (sx, sy, sz) == (0, 0, 0) else -1.0))
        cols, vals = prob.cols[rp[i]:rp[i + 1]], prob.vals[rp[i]:rp[i + 1]]
        got = sorted(zip(cols.tolist(), vals.tolist()))   # oracle columns are global ids
        assert got == sorted(expect), (dims, rank, i)
        assert np.all(vals != 0.0)
