"""paper_conf_sc_luzwflcy0c024_b200 — B200-native (sm_100a) implementation of AmgT's hot
path (Lu et al., SC'24): the mBSR SpGEMM/SpMV kernel pair, CSR<->mBSR conversion, the
per-level precision cast and a fixed-aggregation V-cycle, behind the C ABI in
include/amgt.h (libamgt.so).  This package is the thin Python binding (ctypes).
"""
from ._lib import (  # noqa: F401
    FP16, FP32, FP64, EXPORTED, LIB_PATH, AmgtError, Hierarchy, Mbsr, csr_to_mbsr, from_csr, launch_count, rap,
    set_tc_threshold, SweepPlan, pmis_aggregate, aggregation_p, sa_interp, spgemm, strength_filter, spgemm_numeric, spgemm_symbolic, spmv, spmv_fused, spmv_jacobi_res, timing_enable, timing_read, timing_reset, timing_sample,
    version, wrap,
)
