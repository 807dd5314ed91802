"""bench.py's host-side metrics (no GPU): the overlapped roofline T*_d agrees
with the oracle's definition (oracle/metrics.roofline_tstar), Jain
per reading R-2 reduces to its closed forms, the link-peak helpers never
under-report a peak."""
import types

import pytest

import bench
import strings_workload as W
from oracle import metrics


def _oracle_jobs(wl, kl_slots):
    jobs = []
    for j in wl.jobs:
        if j.kclass == W.GEMM:
            hbm, fl = 2 * j.m * j.k + 2 * j.k * j.n + 4 * j.m * j.n, 2 * j.m * j.n * j.k * j.reps
        elif j.kclass == W.HIST:
            hbm, fl = j.n + 1024, 0
        else:
            hbm, fl = 8 * j.n, 0
        jobs.append({"h2d": sum(j.h2d_sizes()), "d2h": sum(j.d2h_sizes()), "hbm": hbm, "flop": fl,
                     "tenant": j.tenant, "arrival": j.arrival_ns / 1e9, "sms": 148 / kl_slots})
    return jobs


@pytest.mark.parametrize("name,kw", [("C1", {}), ("C2", dict(scale=16)), ("C3", {}), ("C4", dict(scale=8)),
                                     ("C5", dict(scale=16, jobs_per_tenant=6))])
@pytest.mark.parametrize("kl_slots", [1, 2, 8])
def test_tstar_device_matches_the_oracle_definition(name, kw, kl_slots):
    wl = W.CONFIGS[name](**kw)
    h2d, d2h, hbm, tf = 55.0, 57.0, 6500.0, 1400.0
    # bidir = h2d + d2h makes the bench's concurrent-link term never the max (mediant)
    link = {"h2d_gbs": h2d, "d2h_gbs": d2h, "bidir_gbs": h2d + d2h}
    got, terms = bench.tstar_device(wl, link, hbm, tf, kl_slots=kl_slots)
    peaks = {"B_h2d": h2d * 1e9, "B_d2h": d2h * 1e9, "B_hbm": hbm * 1e9, "F_gpu": tf * 1e12, "F_sm": tf * 1e12 / 148}
    t0 = min(j.arrival_ns for j in wl.jobs) / 1e9
    want = metrics.roofline_tstar(_oracle_jobs(wl, kl_slots), peaks, t0=t0)
    assert got == pytest.approx(want, rel=1e-12)
    assert terms["bidir"] <= max(terms["h2d"], terms["d2h"]) * (1 + 1e-12)


def test_tstar_bidir_term_binds_when_the_concurrent_link_is_slower():
    wl = W.config_c2(scale=16)
    link = {"h2d_gbs": 55.0, "d2h_gbs": 57.0, "bidir_gbs": 80.0}
    t, terms = bench.tstar_device(wl, link, 6500.0, 1400.0)
    assert t == terms["bidir"] > max(terms["h2d"], terms["d2h"])


def test_jain_r2_closed_forms():
    wl = W.Workload("j", W.SystemConfig(), [W.TenantSpec(weight=1), W.TenantSpec(weight=2)],
                    [W.JobSpec(tenant=0, kclass=W.VSCALE), W.JobSpec(tenant=1, kclass=W.VSCALE)])
    # x_i = (alone / shared) / w: tenant 1 twice the weight, half the progress -> unequal
    j, xs = bench.jain_r2(wl, {0: 2.0, 1: 4.0}, {0: 1.0, 1: 1.0})
    assert xs == [0.5, 0.125]
    assert j == pytest.approx((0.625 ** 2) / (2 * (0.25 + 0.015625)))
    # equal weighted progress -> 1
    j, _ = bench.jain_r2(wl, {0: 2.0, 1: 1.0}, {0: 1.0, 1: 1.0})
    assert j == pytest.approx(1.0)


def test_mean_latency_by_tenant_counts_from_the_batch_start():
    info = lambda t, arr, done: types.SimpleNamespace(tenant=t, t_arrival=arr, t_done=[0, 0, done])  # noqa: E731
    got = bench.mean_latency_by_tenant([info(0, 1000, 3000), info(0, 1500, 5000), info(1, 1200, 2000)])
    assert got == {0: pytest.approx(3000e-9), 1: pytest.approx(1000e-9)}


def test_link_helpers_never_under_report():
    a = {"h2d_gbs": 50.0, "d2h_gbs": 55.0, "bidir_gbs": 90.0}
    b = {"h2d_gbs": 55.0, "d2h_gbs": 52.0, "bidir_gbs": 99.0}
    assert bench.max_link(a, b) == {"h2d_gbs": 55.0, "d2h_gbs": 55.0, "bidir_gbs": 99.0}
    one = bench.scaled_link(a, {"gpus": 1, "aggregate_bidir_gbs": 95.0, "per_gpu_bidir_gbs": 95.0})
    assert one["bidir_gbs"] == 95.0 and one["h2d_gbs"] == 50.0
    eight = bench.scaled_link(b, {"gpus": 8, "aggregate_bidir_gbs": 8 * 49.5, "per_gpu_bidir_gbs": 49.5})
    assert eight["bidir_gbs"] == pytest.approx(49.5) and eight["h2d_gbs"] == pytest.approx(27.5)
