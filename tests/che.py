"""Closed-form cache pins (test helper; independent of oracle/ and of the CUDA path).

* Che approximation of an LRU cache under the independent-reference model (IRM):
  solve  sum_k s_k (1 - exp(-p_k T)) = C  for the characteristic time T, then
  hit = sum_k p_k (1 - exp(-p_k T))   (per-lookup hit ratio).
  With s_k = row bytes this is the byte-capacity form used for mixed dims.
* IRM static optimum: the C most probable keys' mass (an upper bound on any
  online policy's steady-state hit ratio; SURVEY c-6, reading R19 "Optimal").
* Expected unique keys per batch of N lookups: sum_k (1 - exp(-p_k N)).

Key probabilities: a lookup goes to table t with weight w_t (uniform for one-hot
batches: every sample has one ID per table), then rank r with prob r^-a / H(c, a);
ranks map to rows bijectively so only the multiset of probabilities matters.
"""
from __future__ import annotations

import numpy as np
from scipy.optimize import brentq

_HEAD = 200_000


def _table_probs(c: int, a: float):
    """(probabilities, multiplicities) of one table's ranks; tail of huge tables grouped."""
    c = int(c)
    if c <= _HEAD * 2:
        r = np.arange(1, c + 1, dtype=np.float64)
        w = r ** (-a)
        return w / w.sum(), np.ones(c)
    r = np.arange(1, _HEAD + 1, dtype=np.float64)
    head = r ** (-a)
    # tail ranks (HEAD, c] grouped into log-spaced bins, each bin's ranks share the midpoint prob
    edges = np.unique(np.round(np.geomspace(_HEAD + 1, c + 1, 20000)).astype(np.int64))
    lo, hi = edges[:-1], edges[1:]
    mult = (hi - lo).astype(np.float64)
    mid = (lo + hi - 1) / 2.0
    tail = mid ** (-a)
    H = head.sum() + (tail * mult).sum()
    return np.concatenate([head / H, tail / H]), np.concatenate([np.ones(_HEAD), mult])


def key_probs(cards, skews, weights=None):
    n = len(cards)
    if weights is None:
        weights = [1.0 / n] * n
    ps, ms, ts = [], [], []
    for t, (c, a, w) in enumerate(zip(cards, skews, weights)):
        p, m = _table_probs(c, a)
        ps.append(p * w)
        ms.append(m)
        ts.append(np.full(p.size, t))
    return np.concatenate(ps), np.concatenate(ms), np.concatenate(ts)


def che_hit(cards, skews, cap, sizes=None, weights=None) -> float:
    """Per-lookup steady-state hit ratio of an LRU cache of capacity `cap`.

    cap is in rows when sizes is None, else in bytes with sizes[t] = row bytes of table t."""
    p, m, t = key_probs(cards, skews, weights)
    s = m if sizes is None else m * np.asarray(sizes, dtype=np.float64)[t]
    total = s.sum()
    if cap >= total:
        return 1.0

    def f(logT):
        return (s * -np.expm1(-p * np.exp(logT))).sum() - cap

    logT = brentq(f, -50.0, 80.0, xtol=1e-12)
    T = np.exp(logT)
    return float((m * p * -np.expm1(-p * T)).sum())


def irm_optimum(cards, skews, cap_rows, weights=None) -> float:
    p, m, _ = key_probs(cards, skews, weights)
    order = np.argsort(-p)
    p, m = p[order], m[order]
    cm = np.cumsum(m)
    k = np.searchsorted(cm, cap_rows, side="right")
    mass = (p[:k] * m[:k]).sum()
    if k < p.size:
        mass += p[k] * (cap_rows - (cm[k - 1] if k else 0))
    return float(mass)


def expected_unique(cards, skews, lookups_per_table) -> float:
    n = len(cards)
    p, m, _ = key_probs(cards, skews)
    N = lookups_per_table * n
    return float((m * -np.expm1(-p * N)).sum())
