import sys, os, numpy as np, torch
sys.path.insert(0, os.getcwd())
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
A = gen.irregular_block_sparse(1 << 12, seed=11)
M = amgt.from_csr(A)
C, info = amgt.spgemm(M, M, info=True)
v1 = C.blc_val.clone()
amgt.spgemm_numeric(M, M, C)
v2 = C.blc_val.clone()
d = (v1 - v2).abs().reshape(-1, 16).amax(1)
bad = torch.nonzero(d > 1e-12 * (v1.abs().reshape(-1, 16).amax(1) + 1e-300)).flatten().cpu().numpy()
ptr = C.blc_ptr.cpu().numpy()
rows = np.searchsorted(ptr, bad, side="right") - 1
print("tiles", C.blc_num, "bad tiles", bad.size, "rows", np.unique(rows)[:20], "nC of rows", np.diff(ptr)[np.unique(rows)][:20])
if bad.size:
    q = bad[0]
    print("tile", q, "v1", v1.reshape(-1, 16)[q].cpu().numpy(), "v2", v2.reshape(-1, 16)[q].cpu().numpy(), "map", hex(int(C.map_u16()[q])))
print("bins", info["bin_rows"])
