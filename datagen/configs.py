"""The five BASELINE.json workloads as seeded synthetic recipes.

Each config is a generator recipe (pattern + value kind + N + dtype + seeds),
not data.  Shapes follow the paper's datasets (Table 1) and
the public OGB/Planetoid statistics named in SURVEY.md §8(d); p_local was
calibrated once (tests/tools/calibrate.py) so that MeanNnzTC lands near the target
(Table 2) and then frozen here.
"""
from __future__ import annotations

import dataclasses
import numpy as np

from . import powerlaw_csr, banded_csr, values, zipf_beta_for, STREAM_AVALS, STREAM_B
from . import lib as _lib  # noqa: F401  (ensures the generator builds on import of configs users)


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    desc: str
    kind: str              # "powerlaw" | "banded"
    M: int
    K: int
    nnz: int               # target
    N: int
    dtype: str             # "tf32" | "fp16"
    seed_a: int
    seed_b: int
    # G1
    alpha: float = 2.1
    d_max: int = 0
    p_local: float = 0.5
    S: int = 16
    mean_nnz_tc_target: float = 0.0
    # G2
    per_row: int = 40
    half_band: int = 64
    n_out: int = 8
    out_len: int = 100_000
    gpus: tuple = (1,)
    n_sweep: tuple = ()


CONFIGS: dict[str, Config] = {
    "c1": Config("c1", "Cora-shaped power-law graph", "powerlaw", 2708, 2708, 10556, 32, "tf32",
                 1, 1001, alpha=2.1, d_max=168, p_local=0.6187, S=16, mean_nnz_tc_target=10.0),
    "c2": Config("c2", "ogbn-arxiv-shaped graph", "powerlaw", 169343, 169343, 1166243, 128, "tf32",
                 2, 1002, alpha=2.1, d_max=13161, p_local=0.8662, S=32, mean_nnz_tc_target=10.0),
    "c3": Config("c3", "Reddit-shaped dense-row graph", "powerlaw", 232965, 232965, 114848857, 256,
                 "tf32", 3, 1003, alpha=2.5, d_max=21657, p_local=0.8353, S=1024,
                 mean_nnz_tc_target=16.53, gpus=(1, 8)),
    "c4": Config("c4", "SuiteSparse-shaped banded/FEM matrix with long-row outliers", "banded",
                 1000005, 1000005, 40_800_000, 128, "tf32", 4, 1004, n_sweep=(64, 128, 256)),
    "c5": Config("c5", "ogbn-products-shaped graph", "powerlaw", 2449029, 2449029, 123718280, 512,
                 "tf32", 5, 1005, alpha=2.3, d_max=17481, p_local=0.8044, S=256,
                 mean_nnz_tc_target=12.0, gpus=(1, 2, 4, 8)),
}
# FP16 variant of c3 (same pattern, values rounded to fp16)
CONFIGS["c3h"] = dataclasses.replace(CONFIGS["c3"], name="c3h", dtype="fp16",
                                     desc="Reddit-shaped dense-row graph (FP16 inputs)")


def zipf_beta(cfg: Config) -> float:
    """Zipf exponent so that the hottest column's expected count equals d_max
    (a symmetric-graph proxy: in-degree max ~ out-degree max)."""
    draws = (1.0 - cfg.p_local) * cfg.nnz
    return zipf_beta_for(cfg.K, draws, cfg.d_max)


def make_pattern(cfg: Config, p_local: float | None = None):
    """(rowptr int32[M+1], colidx int32[nnz]) of the config's sparsity pattern."""
    if cfg.kind == "powerlaw":
        pl = cfg.p_local if p_local is None else p_local
        c = dataclasses.replace(cfg, p_local=pl)
        return powerlaw_csr(cfg.M, cfg.K, cfg.nnz, cfg.alpha, cfg.d_max, pl, cfg.S,
                            zipf_beta(c), cfg.seed_a)
    if cfg.kind == "banded":
        return banded_csr(cfg.M, cfg.K, cfg.per_row, cfg.half_band, cfg.n_out, cfg.out_len, cfg.seed_a)
    raise ValueError(cfg.kind)


def make_values(cfg: Config, nnz: int, kind: str = "uniform") -> np.ndarray:
    """A's values: U(-1,1) fp32 (or the pin variants); FP16 configs round to fp16
    and the fp16 array is THE input (its exact fp32 upcast feeds the oracle)."""
    v = values(kind, cfg.seed_a, STREAM_AVALS, nnz)
    return v.astype(np.float16) if cfg.dtype == "fp16" else v


def make_B(cfg: Config, N: int | None = None, kind: str = "uniform") -> np.ndarray:
    """Dense B (K x N) row-major, U(-1,1) (fp16-rounded for FP16 configs)."""
    N = cfg.N if N is None else N
    b = values(kind, cfg.seed_b, STREAM_B, cfg.K * N).reshape(cfg.K, N)
    return b.astype(np.float16) if cfg.dtype == "fp16" else b


def get(name: str) -> Config:
    return CONFIGS[name]
