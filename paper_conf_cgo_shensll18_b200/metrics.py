"""Derived metrics on the library's outputs (host-side
post-processing: "can be built into post processing").

* average reuse distance R.D. over the finite distances (stats["finite_sum"]
  / number of finite accesses), average memory-divergence degree M.D.
  ("average of weighted sum of distribution"), and Eq. (1):

      Opt_Num_Warps = floor( L1_Cache_Size / (R.D. * Cacheline_Size * M.D. * #CTAs/SM) )

  (the number of warps per CTA allowed to use L1 under
  horizontal cache bypassing);
* cross-instance statistics (mean / min / max / stddev of a metric over the
  kernel instances of an application, each analysed separately).
"""
from __future__ import annotations

import math

import numpy as np


def mean_reuse_distance(stats: dict) -> float:
    """R.D.: mean of the finite reuse distances (∞ excluded)."""
    finite = stats["accesses"] - stats["inf"]
    return stats["finite_sum"] / finite if finite else 0.0


def md_degree(hist) -> float:
    """M.D.: sum_k k h_k / sum_k h_k over the (per-kind rows of the) MD histogram."""
    h = np.asarray(hist, dtype=np.float64)
    h = h.reshape(-1, h.shape[-1]).sum(axis=0)
    tot = h.sum()
    return float((h * np.arange(h.size)).sum() / tot) if tot else 0.0


def opt_num_warps(l1_cache_bytes: float, rd: float, line_bytes: float, md: float, ctas_per_sm: float) -> int:
    """Eq. (1) of PAPER.md (L363).  A zero denominator (no reuse or no
    divergence data) leaves L1 to every warp: returns -1."""
    den = rd * line_bytes * md * ctas_per_sm
    return int(math.floor(l1_cache_bytes / den)) if den > 0 else -1


def instance_stats(values) -> dict:
    """Cross-instance mean / min / max / stddev (population) of a metric."""
    v = np.asarray(list(values), dtype=np.float64)
    if v.size == 0:
        return {"n": 0, "mean": 0.0, "min": 0.0, "max": 0.0, "stddev": 0.0}
    return {"n": int(v.size), "mean": float(v.mean()), "min": float(v.min()), "max": float(v.max()),
            "stddev": float(v.std())}
