"""Oracle-backed compute backend for the distributed driver's CPU tests (gloo, world
size 2): exercises the partition / halo / remap / exchange logic of
paper_conf_sc_luzwflcy0c024_b200.dist without a GPU.  Test infrastructure only."""
import numpy as np
import torch

import oracle


class OracleOps:
    device = "cpu"

    def csr_to_local(self, rp, col, val, m, n_cols, col_offset, prec):
        c = (col.numpy().astype(np.int64) - col_offset)
        assert (c >= 0).all() and (c < n_cols).all()
        return oracle.Csr(int(m), int(n_cols), rp.numpy().astype(np.int64).copy(), c.astype(np.int32),
                          val.numpy().astype(np.float64).copy())

    def csr_col_range(self, rp, col, m, row_offset):
        rp, col = rp.numpy(), col.numpy().astype(np.int64)
        mn, mx, bw = np.iinfo(np.int64).max, np.iinfo(np.int64).min, 0
        for i in range(m):
            if rp[i + 1] > rp[i]:
                lo, hi = col[rp[i]], col[rp[i + 1] - 1]
                mn, mx = min(mn, lo), max(mx, hi)
                bw = max(bw, i + row_offset - lo, hi - i - row_offset)
        return int(mn), int(mx), int(bw)

    def col_range_tiles(self, A, blk_row_offset):
        mn, mx, bw = np.iinfo(np.int64).max, np.iinfo(np.int64).min, 0
        for i in range(A.m):
            a, b = A.row_ptr[i], A.row_ptr[i + 1]
            if b > a:
                lo, hi = int(A.col[a]) // 4, int(A.col[b - 1]) // 4
                mn, mx = min(mn, lo), max(mx, hi)
                I = i // 4 + blk_row_offset
                bw = max(bw, I - lo, hi - I)
        return int(mn), int(mx), int(bw)

    def shift_cols(self, A, delta_tiles, new_n):
        return oracle.Csr(A.m, int(new_n), A.row_ptr, (A.col.astype(np.int64) + 4 * delta_tiles).astype(np.int32), A.val)

    def spgemm(self, A, B):
        return oracle.spgemm(A, B)

    def transpose(self, A):
        return oracle.transpose(A)

    def cast(self, A, prec):
        return A

    def to_csr(self, A):
        return torch.from_numpy(A.row_ptr), torch.from_numpy(A.col), torch.from_numpy(A.val)

    def blc_row(self, A):
        return (A.m + 3) // 4

    def spmv_range(self, A, i0, i1, x, y, mode, b=None, dinv=None, xs=None, omega=2.0 / 3.0):
        r0, r1 = 4 * i0, min(4 * i1, A.m)
        if r1 <= r0:
            return y
        rp = A.row_ptr[r0:r1 + 1] - A.row_ptr[r0]
        sub = oracle.Csr(r1 - r0, A.n, rp, A.col[A.row_ptr[r0]:A.row_ptr[r1]], A.val[A.row_ptr[r0]:A.row_ptr[r1]])
        xv = x.double().numpy()
        xv = np.concatenate([xv, np.zeros(max(0, A.n - xv.size))])
        t = oracle.spmv(sub, xv)
        yv = y.numpy()
        if mode == "y":
            yv[r0:r1] = t
        elif mode == "residual":
            yv[r0:r1] = b.numpy()[r0:r1] - t
        elif mode == "accum":
            yv[r0:r1] = yv[r0:r1] + t
        else:
            yv[r0:r1] = xs.numpy()[r0:r1] + omega * dinv.numpy()[r0:r1] * (b.numpy()[r0:r1] - t)
        return y

    def dinv(self, A, diag_tile_offset, dtype):
        d = torch.zeros(4 * ((A.m + 3) // 4), dtype=dtype)
        for i in range(A.m):
            for p in range(A.row_ptr[i], A.row_ptr[i + 1]):
                if A.col[p] == i + 4 * diag_tile_offset:
                    d[i] = 1.0 / A.val[p]
        return d

    def dense_inverse(self, a):
        return np.linalg.inv(a)

    def dense_matvec(self, n, Ainv, b, x):
        x[:n] = Ainv @ b[:n].double()
        return x

    def norm2sq(self, r):
        return torch.tensor([float((r.double() ** 2).sum())], dtype=torch.float64)
