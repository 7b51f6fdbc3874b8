"""ORACLE -- TEST INFRASTRUCTURE ONLY.

Replays of the paper's two strategy selectors on a per-source level profile
(level_sizes[L] = |{v : d(s,v) = L}|, from oracle.single_source).  The mode
decisions are a deterministic function of those sizes, so the
GPU's per-level mode log can be compared with these exactly.

Readings of the garbled/missing algorithm bodies are DESIGN.md §2 R5-R7:

Alg. 4 (hybrid; body missing, caption P:277):
  start with the work-efficient (WE) method for level 0; after level L
  has been expanded, Q_curr_len = |level L|, Q_next_len = |level L+1|,
  Q_change = |Q_next_len - Q_curr_len|; if Q_change > alpha the strategy is
  reconsidered: edge-parallel (EP) iff Q_next_len > beta, else WE; otherwise the
  strategy is kept.  alpha = 768, beta = 512.

Alg. 5 (sampling; body squashed at P:290):
  the first n_samps = 512 sources are processed WE and their maximum BFS depth
  is recorded in keys; keys are sorted and the median keys[n'/2]
  (n' = number of samples) is compared with gamma*log2(n), gamma = 4 (P:290,
  P:299); if smaller, the remaining sources use EP on every level whose frontier
  holds at least 512 vertices, WE otherwise.
"""
from __future__ import annotations

import math
from typing import List, Sequence

WE, EP = 0, 1
ALPHA, BETA = 768, 512
N_SAMPS, GAMMA, EP_MIN_FRONTIER = 512, 4.0, 512


def hybrid_modes(level_sizes: Sequence[int], alpha: int = ALPHA, beta: int = BETA) -> List[int]:
    """Mode used to expand each forward level 0..len-1 under Alg. 4."""
    modes = []
    mode = WE
    for L, q_curr in enumerate(level_sizes):
        modes.append(mode)
        q_next = level_sizes[L + 1] if L + 1 < len(level_sizes) else 0
        if abs(q_next - q_curr) > alpha:
            mode = EP if q_next > beta else WE
    return modes


def sampling_decision(max_depths: Sequence[int], n: int, gamma: float = GAMMA) -> bool:
    """True = edge-parallel run mode.  max_depths are the sampled sources' keys."""
    if len(max_depths) == 0:
        return False
    keys = sorted(max_depths)
    median = keys[len(keys) // 2]
    return median < gamma * math.log2(n)


def sampling_modes(level_sizes: Sequence[int], ep_run: bool,
                   ep_min_frontier: int = EP_MIN_FRONTIER) -> List[int]:
    """Per-level modes for a non-sample source under Alg. 5 with the P:301 guard."""
    if not ep_run:
        return [WE] * len(level_sizes)
    return [EP if q >= ep_min_frontier else WE for q in level_sizes]
