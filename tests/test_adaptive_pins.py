"""Pins of the adaptive-Delta oracle (NEXT-1, PAPER Eq. (1)-(2))
against what the paper states in prose, and a hand-worked example. CPU only."""
import math

import pytest

import oracle


def test_first_two_buckets_fixed():
    # "The Delta_0 and Delta_1 value of the first and second buckets are fixed."
    d = oracle.adaptive_delta([5, 900], [3, 700], 25)
    assert d[0] == 25 and d[1] == 25


@pytest.mark.parametrize("reading", ["A", "B"])
def test_sign_rule(reading):
    # "As the utilization of GPU increases, we reduce Delta_i value, otherwise we
    # increase Delta_i value"; threads stand for utilization.
    up = oracle.adaptive_delta([100, 400], [10, 90], 25, reading)
    down = oracle.adaptive_delta([100, 400], [90, 10], 25, reading)
    assert up[2] < 25 < down[2]


def test_equal_converged_counts_keep_delta():
    # |C_{i-2} - C_{i-1}| = 0 zeroes eps_i whatever the thread counts do.
    d = oracle.adaptive_delta([300, 300, 300], [1, 1000, 5], 16)
    assert d == [16.0, 16.0, 16.0, 16.0]


def test_hand_worked_example():
    # C = (100, 300), T = (50, 150), Delta_0 = 25:
    # eps_2 = (200/400) * (-100/200) * 25 = -6.25 -> Delta_2 = 18.75 (both readings).
    # Then C_2 = 300, T_2 = 100: eps_3 = 0 * ... = 0 (C_1 = C_2) -> A keeps 18.75, B returns to 25.
    a = oracle.adaptive_delta([100, 300, 300], [50, 150, 100], 25, "A")
    b = oracle.adaptive_delta([100, 300, 300], [50, 150, 100], 25, "B")
    assert a == [25.0, 25.0, 18.75, 18.75]
    assert b == [25.0, 25.0, 18.75, 25.0]


def test_eps_bounded_by_delta0():
    # each factor of Eq. (1) is in [-1, 1], so |eps_i| <= Delta_0
    import random

    rng = random.Random(1)
    for _ in range(500):
        C = [rng.randint(0, 10**6) for _ in range(6)]
        T = [rng.randint(0, 10**6) for _ in range(6)]
        d = oracle.adaptive_delta(C, T, 10.0, "B", lo=-math.inf, hi=math.inf)
        assert all(abs(x - 10.0) <= 10.0 + 1e-12 for x in d)


def test_fig6_boundaries_reading_b():
    # Fig. 6 text: with Delta_0 = 25 bucket k ends at 25 (k+1) + sum_{i<=k} eps_i.
    C, T = [10, 50, 20, 80, 40], [5, 30, 60, 10, 20]
    d = oracle.adaptive_delta(C, T, 25, "B", lo=-math.inf, hi=math.inf)
    eps = [x - 25 for x in d]
    end = 0.0
    for k in range(len(d)):
        end += d[k]
        assert math.isclose(end, 25 * (k + 1) + sum(eps[: k + 1]))


def test_clamp():
    d = oracle.adaptive_delta([1, 10**6] * 4, [10**6, 1] * 4, 8, "A")
    assert max(d) <= 32 and min(d) >= 2
