"""Latency metrics (reading R25): the oracle's definitions
pinned by textbook nearest-rank examples and the hand-worked deviation
fixture E6, then the product's reporting module checked against the oracle."""
import random

import pytest

from oracle import metrics_ref as M
from paper_conf_eurosys_zhangcc0xz0g25_b200 import metrics as P
from tests.helpers import load_golden

FX = load_golden("e6_metrics.json")


@pytest.mark.parametrize("case", FX["nearest_rank"])
def test_oracle_nearest_rank_textbook(case):
    for p, want in case["p"].items():
        assert M.percentile(case["xs"], float(p)) == want
        # order of the sample must not matter
        assert M.percentile(list(reversed(case["xs"])), float(p)) == want


def _means(d):
    return {int(j): M.mean(v) for j, v in d.items()}


@pytest.mark.parametrize("qa", FX["quota_assignments"], ids=lambda q: q["label"])
def test_oracle_deviation_and_attainment_fixture(qa):
    iso = {int(j): v for j, v in qa["iso_ms"].items()}
    sysm = _means(qa["sys_latencies_ms"])
    assert M.deviation(sysm, iso) == pytest.approx(qa["expected"]["deviation"], abs=1e-12)
    for j, want in qa["expected"]["attainment"].items():
        assert M.attainment(iso[int(j)], sysm[int(j)]) == pytest.approx(want, rel=1e-12)


def test_oracle_average_deviation_fixture():
    devs = []
    for qa in FX["quota_assignments"]:
        devs.append(M.deviation(_means(qa["sys_latencies_ms"]), {int(j): v for j, v in qa["iso_ms"].items()}))
    assert M.average_deviation(devs) == pytest.approx(FX["expected_average_deviation"], abs=1e-12)


def test_oracle_deviation_invariants():
    rnd = random.Random(5)
    for _ in range(200):
        n = rnd.randint(1, 6)
        iso = {j: rnd.uniform(1, 10) for j in range(n)}
        sysm = {j: rnd.uniform(1, 10) for j in range(n)}
        d = M.deviation(sysm, iso)
        assert d >= 0
        # a system at or below ISO everywhere has zero deviation (L336: "shorter than ISO")
        assert M.deviation({j: min(sysm[j], iso[j]) for j in iso}, iso) == 0
        # the deviation is the sum of the per-application excesses: adding one
        # application that misses ISO by x raises it by exactly x
        x = rnd.uniform(0.1, 5)
        s2, i2 = dict(sysm), dict(iso)
        s2[n], i2[n] = 3.0 + x, 3.0
        assert M.deviation(s2, i2) == pytest.approx(d + x)


def test_product_metrics_match_oracle():
    rnd = random.Random(11)
    for _ in range(100):
        xs = [rnd.randint(1, 10_000_000) for _ in range(rnd.randint(1, 300))]
        for p in (1, 25, 50, 90, 99, 100):
            assert P.nearest_rank(xs, p) == M.percentile(xs, p)
        s = P.summary_ms(xs)
        assert s["mean_ms"] == pytest.approx(M.mean(xs) / 1e6, rel=1e-12)
        assert s["p50_ms"] == M.percentile(xs, 50) / 1e6
        assert s["p99_ms"] == M.percentile(xs, 99) / 1e6
        n = rnd.randint(1, 5)
        iso = {j: rnd.uniform(1, 10) for j in range(n)}
        sysm = {j: rnd.uniform(1, 10) for j in range(n)}
        assert P.latency_deviation(sysm, iso) == pytest.approx(M.deviation(sysm, iso), abs=1e-12)
        for j in range(n):
            assert P.attainment_pct(iso[j], sysm[j]) == pytest.approx(M.attainment(iso[j], sysm[j]))
    for qa in FX["quota_assignments"]:
        iso = {int(j): v for j, v in qa["iso_ms"].items()}
        sysm = {int(j): sum(v) / len(v) for j, v in qa["sys_latencies_ms"].items()}
        assert P.latency_deviation(sysm, iso) == pytest.approx(qa["expected"]["deviation"], abs=1e-12)
    assert P.average_deviation([1.0, 5.0]) == FX["expected_average_deviation"]
