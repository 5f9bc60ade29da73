"""Pins of the schedule oracle (oracle/schedule.py) -- Algorithm 1.

* the paper's worked example, Fig. 7 (tests/golden/fig7_schedule.json):
  K=2, GPU 1: 1F1B stashes 2, advance forward stashes 3 = 3/8 of AFAB.
* the 1F1B bound "up to K-k+1 micro-batches" on GPU k.
* the textbook special cases: AFAB (GPipe) = all F then all B;
  1F1B (PipeDream-Flush / DAPPLE) = warm-up K-k forwards, steady F/B pairs,
  cool-down backwards.
* validity: each list is a permutation of {F(j), B(j)} with F(j) before B(j),
  forwards and backwards each in micro-batch order.
* joint feasibility by brute-force simulation (reading c16).
"""
import itertools
import json
import os

import pytest

from oracle.schedule import (advance_forward_schedule, default_advance, one_f_one_b_advance,
                             peak_in_flight, simulate_pipeline)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig7_schedule.json")


def test_fig7_worked_example():
    g = json.load(open(GOLDEN))
    K, k, M = g["K"], g["gpu_k"], g["M"]
    a_1f1b = one_f_one_b_advance(K, k)
    assert a_1f1b == g["one_f_one_b_advance_gpu1"]
    assert peak_in_flight(advance_forward_schedule(K, M, k, a_1f1b)) == g["one_f_one_b_peak_stash_gpu1"]
    adv = advance_forward_schedule(K, M, k, a_1f1b + 1)      # one micro-batch forwarded in advance
    assert peak_in_flight(adv) == g["advance_forward_peak_stash_gpu1"]
    afab = advance_forward_schedule(K, M, k, M)
    assert peak_in_flight(afab) == g["afab_peak_stash"]
    num, den = g["advance_forward_over_afab"]
    assert peak_in_flight(adv) * den == peak_in_flight(afab) * num


@pytest.mark.parametrize("K,M", [(2, 8), (4, 8), (4, 16), (8, 64), (6, 3)])
def test_one_f_one_b_bound(K, M):
    for k in range(1, K + 1):
        ops = advance_forward_schedule(K, M, k, one_f_one_b_advance(K, k))
        assert peak_in_flight(ops) == min(K - k + 1, M)
    # P:132 example list [4,3,2,1] for K=4, M=8
    if (K, M) == (4, 8):
        assert [peak_in_flight(advance_forward_schedule(4, 8, k, 4 - k)) for k in range(1, 5)] == [4, 3, 2, 1]


def _textbook_afab(M):
    return [("F", j) for j in range(M)] + [("B", j) for j in range(M)]


def _textbook_1f1b(K, M, k):
    warm = min(K - k, M)
    ops = [("F", j) for j in range(warm)]
    f, b = warm, 0
    while f < M:
        ops.append(("F", f)); f += 1
        ops.append(("B", b)); b += 1
    ops += [("B", j) for j in range(b, M)]
    return ops


@pytest.mark.parametrize("K,M", [(1, 1), (2, 8), (3, 5), (4, 4), (5, 12), (8, 3)])
def test_textbook_special_cases(K, M):
    for k in range(1, K + 1):
        assert advance_forward_schedule(K, M, k, M) == _textbook_afab(M)
        assert advance_forward_schedule(K, M, k, M + 7) == _textbook_afab(M)   # clamp (c15)
        assert advance_forward_schedule(K, M, k, K - k) == _textbook_1f1b(K, M, k)


def test_validity_exhaustive_small():
    for K in range(1, 7):
        for M in range(0, 10):
            for k in range(1, K + 1):
                for a in range(-1, M + 2):
                    ops = advance_forward_schedule(K, M, k, a)
                    assert len(ops) == 2 * M
                    assert sorted(ops) == sorted([("F", j) for j in range(M)] + [("B", j) for j in range(M)])
                    pos = {op: i for i, op in enumerate(ops)}
                    assert all(pos[("F", j)] < pos[("B", j)] for j in range(M))
                    assert [j for kind, j in ops if kind == "F"] == list(range(M))
                    assert [j for kind, j in ops if kind == "B"] == list(range(M))
                    assert peak_in_flight(ops) == (min(max(a, 0) + 1, M) if M else 0)


def test_feasibility_rule_by_simulation():
    """c16: per-GPU advance vectors run without deadlock iff
    min(a_k + 1, M) >= min(a_{k+1} + 1, M) for all k."""
    for K in range(1, 5):
        for M in range(1, 6):
            for adv in itertools.product(range(0, M + 1), repeat=K):
                ok = simulate_pipeline(K, M, adv)["ok"]
                rule = all(min(adv[k] + 1, M) >= min(adv[k + 1] + 1, M) for k in range(K - 1))
                assert ok == rule, (K, M, adv)


def test_default_advance_is_feasible():
    for K in range(1, 7):
        for M in range(1, 9):
            for e in range(0, 4):
                adv = [default_advance(K, M, k, e) for k in range(1, K + 1)]
                assert simulate_pipeline(K, M, adv)["ok"]


# ---------------------------------------------------------------- Alg. 1 lines 9-10 (row f2)
from oracle.schedule import AdvanceController  # noqa: E402


def test_controller_starts_at_1f1b_and_grows_to_afab():
    ctl = AdvanceController(K=4, M=8)
    assert ctl.advance_num == 3                                      # line 1: K-1 (1F1B)
    assert [ctl.advance_for(k) for k in range(1, 5)] == [3, 2, 1, 0]
    t = 10.0
    for expect in [4, 5, 6, 7, 8, 8, 8]:                             # always faster, plenty of memory
        t -= 1.0
        assert ctl.update(t, peak_mem=1.0, mem_per_microbatch=0.1, mem_limit=100.0) == expect
    assert peak_in_flight(advance_forward_schedule(4, 8, 1, ctl.advance_for(1))) == 8   # AFAB


def test_controller_stops_at_the_memory_limit():
    ctl = AdvanceController(K=2, M=8)
    per_mb, limit = 1.0, 5.0
    t = 100.0
    for _ in range(10):
        peak = per_mb * peak_in_flight(advance_forward_schedule(2, 8, 1, ctl.advance_num))
        t -= 1.0
        ctl.update(t, peak, per_mb, limit)
    # stash = advance + 1 micro-batches; growth stops once one more would exceed the limit
    assert ctl.advance_num == 4
    assert peak_in_flight(advance_forward_schedule(2, 8, 1, ctl.advance_num)) * per_mb == limit


def test_controller_holds_when_not_faster():
    ctl = AdvanceController(K=3, M=16)
    assert ctl.advance_num == 2
    # first batch counts as faster -> 3; 9 < 10 -> 4; 9.5 not faster; 9.5 not < 9.5; 8 < 9.5 -> 5; 8 not < 8
    for t, expect in [(10.0, 3), (9.0, 4), (9.5, 4), (9.5, 4), (8.0, 5), (8.0, 5)]:
        assert ctl.update(t, 0.0, 1.0, 1e9) == expect
