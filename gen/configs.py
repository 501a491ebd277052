"""The five BASELINE.json workloads as generator recipes.

`full` sizes are BASELINE's; `small` variants keep the same structure at sizes the
oracle finishes in seconds while still spanning many tiles and ragged tails.
"""
from __future__ import annotations

from dataclasses import dataclass, field


@dataclass(frozen=True)
class Config:
    key: str
    kind: str               # "5pt", "7pt", "27pt", "irregular"
    N: int = 0              # grid points per dimension (stencils)
    BR: int = 0             # block rows (irregular)
    nlev: int = 1           # AMG levels for V-cycle configs
    alpha: float = 0.5      # aggregation value
    seed: int = 0
    description: str = ""
    level_prec: tuple = field(default=("f64", "f32", "f16", "f16", "f16", "f16", "f16"))


CONFIGS = {
    "cfg1": Config("cfg1", "5pt", N=64, nlev=1, alpha=1.0, seed=1,
                   description="2D 5-point Poisson 64x64 (4,096 rows): mBSR A*A SpGEMM + FP64 SpMV"),
    "cfg2": Config("cfg2", "7pt", N=128, nlev=7, alpha=0.5, seed=2,
                   description="3D 7-point Laplacian 128^3: RAP with 2x2x2 aggregation P + FP64/FP32 SpMV"),
    "cfg3": Config("cfg3", "27pt", N=256, nlev=7, alpha=0.5, seed=3,
                   description="3D 27-point Laplacian 256^3: mixed-precision V-cycle"),
    "cfg4": Config("cfg4", "irregular", BR=1 << 18, seed=20240917,
                   description="irregular power-law block-sparse (2^18 block rows): bins + TC/CUDA-core routing"),
    "cfg5": Config("cfg5", "7pt", N=512, nlev=7, alpha=0.5, seed=5,
                   description="3D 7-point Laplacian 512^3 row-partitioned over 2/4/8 GPUs"),
}

SMALL = {
    "cfg1": CONFIGS["cfg1"],
    "cfg2": Config("cfg2s", "7pt", N=24, nlev=4, alpha=0.5, seed=2, description="7-point 24^3"),
    "cfg3": Config("cfg3s", "27pt", N=16, nlev=4, alpha=0.5, seed=3, description="27-point 16^3"),
    "cfg4": Config("cfg4s", "irregular", BR=1 << 11, seed=20240917, description="irregular 2^11 block rows"),
    "cfg5": Config("cfg5s", "7pt", N=32, nlev=4, alpha=0.5, seed=5, description="7-point 32^3"),
}


def build_matrix(cfg: Config, device="cpu", spd_seed=None):
    from .stencils import laplacian_5pt, laplacian_7pt, laplacian_27pt
    from .irregular import irregular_block_sparse
    if cfg.kind == "5pt":
        return laplacian_5pt(cfg.N, device, spd_seed)
    if cfg.kind == "7pt":
        return laplacian_7pt(cfg.N, device, spd_seed)
    if cfg.kind == "27pt":
        return laplacian_27pt(cfg.N, device, spd_seed)
    if cfg.kind == "irregular":
        return irregular_block_sparse(cfg.BR, seed=cfg.seed).to(device)
    raise ValueError(cfg.kind)


def grid_dims(cfg: Config):
    if cfg.kind == "5pt":
        return (cfg.N, cfg.N)
    return (cfg.N, cfg.N, cfg.N)
