"""Helpers for distribution pins: exact laws by enumeration + chi-square."""
from __future__ import annotations

import itertools
from collections import Counter

import numpy as np
from scipy import stats


def chi_square_p(observed: Counter, expected_prob: dict, n: int) -> float:
    keys = sorted(expected_prob)
    extra = set(observed) - set(keys)
    assert not extra, f"outcomes outside the support: {sorted(extra)[:5]}"
    obs = np.array([observed.get(k, 0) for k in keys], dtype=np.float64)
    exp = np.array([expected_prob[k] * n for k in keys], dtype=np.float64)
    assert abs(exp.sum() - n) < 1e-6 * n, "expected law does not sum to 1"
    return float(stats.chisquare(obs, exp).pvalue)


def successive_sampling_law(weights, k):
    """P(S) for weighted sampling without replacement, k successive draws each
    proportional to weight among the remaining items (the law A-Res realises;
    Efraimidis & Spirakis 2006).  Enumerated over ordered k-tuples."""
    n = len(weights)
    W = float(sum(weights))
    law = Counter()
    for tup in itertools.permutations(range(n), k):
        p, rem = 1.0, W
        for i in tup:
            p *= weights[i] / rem
            rem -= weights[i]
        law[tuple(sorted(tup))] += p
    return dict(law)
