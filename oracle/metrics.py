"""Evaluation metrics and the overlapped roofline (reference definitions).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

* Weighted speedup, Eq. (2) (formula glyphs lost):
  reading R-1, WS = (1/N) * sum_i  Tbar_i^base / Tbar_i^policy, Tbar = mean
  completion latency (done - arrival) of tenant i's jobs.  The Snavely-Tullsen
  form [22] sum_i Tbar_i^alone / Tbar_i^shared is ``snavely_tullsen``.
* Jain's fairness, Eq. (3) (glyphs lost):
  reading R-2, J = (sum x)^2 / (N * sum x^2), x_i = normalised progress / w_i.
* Overlapped multi-resource roofline T*_d per device.
"""
from __future__ import annotations

from typing import Dict, Iterable, List, Sequence


def jain(xs: Sequence[float]) -> float:
    xs = [float(x) for x in xs]
    n = len(xs)
    s2 = sum(x * x for x in xs)
    if n == 0 or s2 == 0.0:
        return 1.0
    return sum(xs) ** 2 / (n * s2)


def weighted_speedup(base_lat: Sequence[float], policy_lat: Sequence[float]) -> float:
    assert len(base_lat) == len(policy_lat) and len(base_lat) > 0
    return sum(b / p for b, p in zip(base_lat, policy_lat)) / len(base_lat)


def snavely_tullsen(alone_lat: Sequence[float], shared_lat: Sequence[float]) -> float:
    return sum(a / s for a, s in zip(alone_lat, shared_lat))


def mean_latency_per_tenant(records: Iterable[dict], num_tenants: int) -> List[float]:
    """records: dicts with tenant, arrival, done (ns)."""
    acc = [0.0] * num_tenants
    cnt = [0] * num_tenants
    for r in records:
        acc[r["tenant"]] += r["done"] - r["arrival"]
        cnt[r["tenant"]] += 1
    return [a / c if c else 0.0 for a, c in zip(acc, cnt)]


def roofline_tstar(jobs: List[dict], peaks: Dict[str, float], t0: float = 0.0,
                   inflight: Dict[int, int] = None) -> float:
    """T*_d (seconds) for the jobs placed on one device.

    jobs: dicts with h2d, d2h, hbm (bytes), flop, tenant, arrival (s), sms.
    peaks: B_h2d, B_d2h, B_hbm (bytes/s), F_gpu, F_sm (FLOP/s).
    """
    inflight = inflight or {}
    if not jobs:
        return 0.0
    bh, bd, bm = peaks["B_h2d"], peaks["B_d2h"], peaks["B_hbm"]
    fg, fs = peaks["F_gpu"], peaks["F_sm"]

    def klstar(j):
        f = min(fg, j.get("sms", 148) * fs)
        return max(j["hbm"] / bm, j["flop"] / f if j["flop"] else 0.0)

    terms = [
        sum(j["h2d"] for j in jobs) / bh,
        sum(j["d2h"] for j in jobs) / bd,
        sum(j["hbm"] + j["h2d"] + j["d2h"] for j in jobs) / bm,
        sum(j["flop"] for j in jobs) / fg,
    ]
    chains: Dict[int, float] = {}
    for j in jobs:
        chains[j["tenant"]] = chains.get(j["tenant"], 0.0) + j["h2d"] / bh + klstar(j) + j["d2h"] / bd
    terms.append(max(v / inflight.get(t, 1) for t, v in chains.items()))
    terms.append(max(j.get("arrival", 0.0) + j["h2d"] / bh + klstar(j) + j["d2h"] / bd for j in jobs) - t0)
    return max(terms)
