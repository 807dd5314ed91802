"""Pins for metrics, Eq. (4) generator and brute force (no GPU)."""
import math

import numpy as np
import pytest

import strings_workload as W
from oracle import bruteforce, metrics


def test_jain_limits_and_scale_invariance():
    assert metrics.jain([3, 3, 3, 3]) == pytest.approx(1.0)
    assert metrics.jain([5, 0, 0, 0]) == pytest.approx(0.25)        # 1/N
    xs = [1.0, 2.0, 7.5]
    assert metrics.jain(xs) == pytest.approx(metrics.jain([10 * x for x in xs]))
    assert 1 / 3 <= metrics.jain(xs) <= 1.0
    assert metrics.jain([1, 2]) == pytest.approx(9 / 10)             # (1+2)^2 / (2*5)


def test_weighted_speedup_identity_and_scaling():
    lat = [1.0, 2.0, 3.0]
    assert metrics.weighted_speedup(lat, lat) == pytest.approx(1.0)
    assert metrics.weighted_speedup(lat, [x / 2 for x in lat]) == pytest.approx(2.0)
    assert metrics.snavely_tullsen(lat, lat) == pytest.approx(3.0)


def test_roofline_terms():
    pk = dict(B_h2d=50e9, B_d2h=50e9, B_hbm=6e12, F_gpu=1e15, F_sm=1e13)
    j = dict(h2d=50e6, d2h=25e6, hbm=0.0, flop=0.0, tenant=0)
    # one tenant, two identical jobs: chain = 2*(1ms + 0.5ms) = 3 ms dominates
    assert metrics.roofline_tstar([j, dict(j)], pk) == pytest.approx(3e-3)
    # two tenants: link bound 2 ms
    assert metrics.roofline_tstar([j, dict(j, tenant=1)], pk) == pytest.approx(2e-3)
    # HBM carries the copies too: 1 GB/s of HBM, 1 + 0.5 MB copied -> 1.5 ms (> the 1 ms link term)
    slow_hbm = dict(pk, B_hbm=1e9)
    k = dict(h2d=1e6, d2h=5e5, hbm=0.0, flop=0.0, tenant=0)
    assert metrics.roofline_tstar([k, dict(k, tenant=1)], slow_hbm) == pytest.approx(3e-3)
    # open-loop arrival bound: a job arriving at 10 ms finishes no earlier than 10 ms + its chain
    late = dict(j, arrival=10e-3)
    assert metrics.roofline_tstar([dict(j, tenant=1), late], pk, t0=0.0) == pytest.approx(10e-3 + 1.5e-3)


# ---------------------------------------------------------------- Eq. (4)
def test_eq4_sample_mean_and_x_equal_one():
    rng = W.SplitMix64(123)
    lam = 1_000_000.0
    xs = [W.exp_interarrival_ns(rng, lam) for _ in range(200_000)]
    assert abs(np.mean(xs) / lam - 1.0) < 0.01
    class One:
        def unit_open0(self):
            return 1.0
    assert W.exp_interarrival_ns(One(), lam) == 0          # X = 1 -> T = 0


def test_eq4_memoryless():
    rng = W.SplitMix64(99)
    lam = 1000.0
    xs = np.array([W.exp_interarrival_ns(rng, lam) for _ in range(200_000)], dtype=np.float64)
    s = 700.0
    tail = xs[xs > s] - s
    # P(T > s + t | T > s) = P(T > t): compare quantiles of the residual with the whole
    for q in (0.25, 0.5, 0.75, 0.9):
        assert abs(np.quantile(tail, q) - np.quantile(xs, q)) / lam < 0.03


def test_splitmix64_reference_values():
    # Reference outputs of SplitMix64 seeded with 1234567 (Vigna's splitmix64.c)
    r = W.SplitMix64(1234567)
    assert [r.next_u64() for _ in range(3)] == [6457827717110365317, 3203168211198807973,
                                                9817491932198370423]


def test_unit_open0_range():
    r = W.SplitMix64(0)
    for _ in range(10000):
        x = r.unit_open0()
        assert 0.0 < x <= 1.0


# ------------------------------------------------------------- brute force
def test_bruteforce_small_cases():
    loads = [[3], [3], [2], [2], [2]]          # classic: greedy LPT 7 vs OPT 6
    opt, pl = bruteforce.optimal_vector_load(loads, 2)
    assert opt == 6
    assert bruteforce.vector_load(loads, pl, 2) == 6
    loads2 = [[5, 0], [0, 5], [5, 0], [0, 5]]
    assert bruteforce.optimal_vector_load(loads2, 2)[0] == 5
