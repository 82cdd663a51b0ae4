"""Serving metrics (oracle; test infrastructure only).

PAPER.md §4.1 Metrics: latency = pending time + CUDA execution time,
i.e. finish - arrival; throughput = requests handled per unit time.  Readings
(R18-R20): throughput = completed / (last finish - first arrival);
p99 by nearest rank over all completed requests.
"""
import math


def latencies(arrivals, finishes):
    return [f - a for a, f in zip(arrivals, finishes)]


def mean(xs):
    return sum(xs) / len(xs)


def p_nearest_rank(xs, p):
    s = sorted(xs)
    k = max(1, math.ceil(p / 100.0 * len(s)))
    return s[k - 1]


def throughput(arrivals, finishes, weights=None):
    """Completed units per second; `weights` = sequences per batch (req/s) or 1."""
    n = sum(weights) if weights is not None else len(finishes)
    return n / (max(finishes) - min(arrivals))
