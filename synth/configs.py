"""The five BASELINE.json configs as synthetic-input recipes.

Vertex / edge counts and feature dims follow PAPER.md Table 4; Reddit uses the DGL
edge count (~114.6 M).  Seeds: graph 1, partition 101, emb 3, grad 4.
"""
from dataclasses import dataclass, field
from typing import Tuple


@dataclass(frozen=True)
class Config:
    name: str
    n: int
    e: int
    m: int
    dims: Tuple[int, ...]
    topology: str = "uniform_nvswitch"
    backward_layers: Tuple[int, ...] = ()
    graph_seed: int = 1
    part_seed: int = 101
    emb_seed: int = 3
    grad_seed: int = 4


CONFIGS = {
    # configs[0]: tiny synthetic graph, random 2-way partition, dim 16, one GCN layer exchange
    "tiny": Config("tiny", 10_000, 100_000, 2, (16,), backward_layers=(0,)),
    # configs[1]: Reddit-shaped, 8-way, dim 602 input / 256 hidden.  One GCN training step
    # exchanges both layers forward and layer 1 backward (no gradient w.r.t. input features).
    "reddit": Config("reddit", 232_965, 114_615_892, 8, (602, 256), backward_layers=(1,)),
    # configs[2]: Web-Google-shaped, dim 256, 2/4/8-way
    "google2": Config("google2", 875_713, 5_105_039, 2, (256,), backward_layers=(0,)),
    "google4": Config("google4", 875_713, 5_105_039, 4, (256,), backward_layers=(0,)),
    "google8": Config("google8", 875_713, 5_105_039, 8, (256,), backward_layers=(0,)),
    # configs[3]: Com-Orkut-shaped, dim 128, 8-way, forward + backward per layer
    "orkut": Config("orkut", 3_072_441, 117_185_083, 8, (128,), backward_layers=(0,)),
    # configs[4]: forced non-uniform topology models on 8 GPUs (relay hops)
    "google8_dgx1": Config("google8_dgx1", 875_713, 5_105_039, 8, (256,), topology="dgx1_like",
                           backward_layers=(0,)),
    "google8_ring": Config("google8_ring", 875_713, 5_105_039, 8, (256,), topology="ring",
                           backward_layers=(0,)),
    "reddit_dgx1": Config("reddit_dgx1", 232_965, 114_615_892, 8, (256,), topology="dgx1_like",
                          backward_layers=(0,)),
}


def get_config(name):
    return CONFIGS[name]


def pitch_of(dim):
    """Harness row pitch: dim rounded up to a multiple of 4 floats (16-B rows)."""
    return (dim + 3) // 4 * 4
