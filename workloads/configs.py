"""The five BASELINE.json configs as synthetic inputs (SURVEY.md §8(d) "Structure per config").

Comm models are assumptions (Fig. 4(b) values are not extractable from PAPER.md L138):
  NVLink-V100-like: beta0 = 10,000 ns, beta1 = 40,000 fs/B (25 GB/s per direction)
  comm-heavy:       beta1 = 400,000 fs/B (0.1x, "on the order of PCIe")
"""

from __future__ import annotations

from dataclasses import dataclass
from functools import lru_cache

from . import dag, shaped

NVLINK_BETA0 = 10_000
NVLINK_BETA1 = 40_000
HEAVY_BETA1 = 400_000

SEARCH_SEED = 2021
MOVE_MIX = (50, 20, 20, 10)      # FLIP1, FLIPk, WINDOW (lane-level weights), SWAP (% of warps)


@dataclass(frozen=True)
class Config:
    name: str
    graph: str               # generator name
    D: int
    beta0: int
    beta1: int
    candidates_per_gpu: int  # K per GPU per search step (all bases together)
    bases: int = 4
    oracle_sample: int = 2048


CONFIGS = {
    "tiny12": Config("tiny12", "tiny12", 2, 1000, 1_000_000, 4096, 1, 761_856),
    "inception_v3_2dev": Config("inception_v3_2dev", "inception_v3", 2, NVLINK_BETA0,
                                NVLINK_BETA1, 65_536, 4, 4096),
    "nmt4_2dev_commheavy": Config("nmt4_2dev_commheavy", "nmt", 2, NVLINK_BETA0, HEAVY_BETA1,
                                  262_144, 4, 1024),
    "transformer_2dev": Config("transformer_2dev", "transformer", 2, NVLINK_BETA0, NVLINK_BETA1,
                               1_048_576, 4, 2048),
    "transformer_4dev_8gpu": Config("transformer_4dev_8gpu", "transformer", 4, NVLINK_BETA0,
                                    NVLINK_BETA1, 1_048_576, 4, 2048),
}


@lru_cache(maxsize=8)
def _base_graph(kind: str) -> dag.Graph:
    if kind == "tiny12":
        return dag.tiny12()
    if kind == "inception_v3":
        return shaped.inception_v3()
    if kind == "nmt":
        return shaped.nmt()
    if kind == "transformer":
        return shaped.transformer()
    raise KeyError(kind)


def graph_for(cfg: Config) -> dag.Graph:
    g = _base_graph(cfg.graph)
    return g.with_comm(cfg.D, cfg.beta0, cfg.beta1)
