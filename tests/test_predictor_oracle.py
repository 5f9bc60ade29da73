"""Pins of the tuning-predictor oracle (oracle/predictor.py; §5.2, Eqs. (1)-(8)).

* the paper's own special cases: at (m*, n*) = (m, n) with phi < 1, Eq. (2)
  gives T_gpu, Eq. (4) reduces to Eq. (3), Eq. (8) gives F_mod + F_dat (P:210,
  P:216);
* a closed form from conservation of work: for a constant utilisation phi0
  over a window equal to T_gpu, T_gpu* = max(T_gpu / c, phi0 * T_gpu) with
  c = m n*/(m* n) (linear scaling until the GPU saturates, Fig. 8);
* hand-computed bubble recursions (Eqs. (6)/(7)) and memory (Eq. (8));
* tune() picks a feasible setting no feasible candidate beats.
"""
import itertools

import numpy as np
import pytest

from oracle.predictor import Profile, predict, t_gpu_star, tune


def _profile(K=3, m=8, n=2, S=100, seed=0, phi_max=0.6):
    rng = np.random.default_rng(seed)
    t_gpu = rng.uniform(0.5, 2.0, K)
    return Profile(m=m, n=n, dt=float(t_gpu.mean()) / S, phi=rng.uniform(0.05, phi_max, (K, S)),
                   t_gpu=list(t_gpu), t_comm=list(rng.uniform(0.1, 1.5, K)), f_mod=list(rng.uniform(1e9, 4e9, K)),
                   f_dat=list(rng.uniform(1e9, 8e9, K)))


def test_identity_at_the_profiled_setting():
    prof = _profile()
    p = predict(prof, prof.m, prof.n)
    for k in range(prof.K):
        assert p["t_gpu"][k] == pytest.approx(prof.t_gpu[k], rel=1e-15)
        eq3 = prof.t_comm[k] / prof.m + (prof.m - 1) / prof.m * max(prof.t_comm[k] - prof.t_gpu[k], 0.0)
        assert p["t_com"][k] == pytest.approx(eq3, rel=1e-15)
        assert p["mem"][k] == pytest.approx(prof.f_mod[k] + prof.f_dat[k], rel=1e-15)


@pytest.mark.parametrize("phi0", [0.1, 0.3, 0.5, 0.9])
@pytest.mark.parametrize("m_star,n_star", [(8, 2), (4, 2), (2, 2), (1, 2), (16, 2), (8, 4), (2, 6), (32, 1)])
def test_constant_utilisation_closed_form(phi0, m_star, n_star):
    S, T = 1000, 1.7
    prof = Profile(m=8, n=2, dt=T / S, phi=np.full((1, S), phi0), t_gpu=[T], t_comm=[0.3], f_mod=[1.0],
                   f_dat=[1.0])
    c = (prof.m * n_star) / (m_star * prof.n)
    assert t_gpu_star(prof, 0, m_star, n_star) == pytest.approx(max(T / c, phi0 * T), rel=1e-12)


def test_bubble_recursion_hand_computed():
    # phi = 0 -> no saturation term: T_gpu* = (m* n)/(m n*) T_gpu = T_gpu / 2 at m* = m/2
    prof = Profile(m=4, n=1, dt=1.0, phi=np.zeros((3, 4)), t_gpu=[4.0, 8.0, 12.0], t_comm=[1.0, 1.0, 1.0],
                   f_mod=[10.0, 20.0, 30.0], f_dat=[5.0, 5.0, 5.0])
    p = predict(prof, 2, 1)
    assert p["t_gpu"] == pytest.approx([2.0, 4.0, 6.0])
    # Eq. (6): up = [0, (1+2)/2, 1.5 + (1+4)/2];  Eq. (7): down = [3.5 + (1+4)/2, (1+6)/2, 0]
    assert p["t_up"] == pytest.approx([0.0, 1.5, 4.0])
    assert p["t_down"] == pytest.approx([6.0, 3.5, 0.0])
    # Eq. (4): 1/2 + 1/2 * max(1 - T_gpu*, 0) = 0.5 (T_gpu* > 1 everywhere)
    assert p["t_com"] == pytest.approx([0.5, 0.5, 0.5])
    assert p["t_total"] == pytest.approx([2 + 0.5 + 6.0, 4 + 0.5 + 5.0, 6 + 0.5 + 4.0])
    assert p["iter_time"] == pytest.approx(10.5)
    # Eq. (8): n*/n F_mod + (m n*)/(m* n) F_dat = F_mod + 2 F_dat
    assert p["mem"] == pytest.approx([20.0, 30.0, 40.0])
    p2 = predict(prof, 4, 3)          # three pipelines: F_mod x3, F_dat x3
    assert p2["mem"] == pytest.approx([45.0, 75.0, 105.0])


def test_communication_overlap_term():
    # TT > T_gpu*: every micro-batch after the first is blocked by (TT - T_gpu*)/m*
    prof = Profile(m=4, n=2, dt=0.1, phi=np.zeros((1, 10)), t_gpu=[1.0], t_comm=[3.0], f_mod=[0.0], f_dat=[0.0])
    p = predict(prof, 4, 4)           # n* = 2n: TT* = 6, T_gpu* = 1/2
    assert p["t_gpu"][0] == pytest.approx(0.5)
    assert p["t_com"][0] == pytest.approx(4 / (4 * 2) * 3.0 + 3 / 4 * (6.0 - 0.5))


@pytest.mark.parametrize("seed", range(5))
def test_tune_picks_an_unbeaten_feasible_setting(seed):
    prof = _profile(K=4, seed=seed)
    ms, ns = [1, 2, 4, 8, 16, 32], [1, 2, 3, 4]
    limit = float(np.median([predict(prof, m, n)["peak_mem"] for m, n in itertools.product(ms, ns)]))
    res = tune(prof, ms, ns, limit)
    assert res is not None
    m_b, n_b, t_b = res
    pb = predict(prof, m_b, n_b)
    assert pb["peak_mem"] <= limit
    for m, n in itertools.product(ms, ns):
        p = predict(prof, m, n)
        if p["peak_mem"] <= limit:
            assert n / p["iter_time"] <= n_b / t_b * (1 + 1e-12)
    assert tune(prof, ms, ns, 0.0) is None
    m_t, n_t, t_t = tune(prof, ms, ns, limit, objective="time")
    assert all(predict(prof, m, n)["iter_time"] >= t_t * (1 - 1e-12)
               for m, n in itertools.product(ms, ns) if predict(prof, m, n)["peak_mem"] <= limit)
