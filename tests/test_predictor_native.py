"""Native tuning predictor (ea_predict / ea_tune, row f3) vs the oracle
(oracle/predictor.py) on random profiles: predictions within 1e-12 relative,
the chosen setting identical (an integer decision both sides take in double)."""
import itertools

import numpy as np
import pytest

from oracle.predictor import Profile, predict as o_predict, tune as o_tune
from paper_conf_ppopp_chen0qz23_b200 import binding
from paper_conf_ppopp_chen0qz23_b200.build import build


@pytest.fixture(scope="module", autouse=True)
def lib():
    build()
    return binding.load_library()


def _rand(seed, K=None, S=None):
    rng = np.random.default_rng(seed)
    K = K or int(rng.integers(1, 9))
    S = S if S is not None else int(rng.integers(0, 200))
    t_gpu = rng.uniform(0.01, 3.0, K)
    return dict(m=int(rng.integers(1, 64)), n=int(rng.integers(1, 5)), dt=float(rng.uniform(1e-4, 0.05)),
                phi=rng.uniform(0.0, 1.0, (K, S)) * rng.uniform(0.2, 1.0), t_gpu=t_gpu,
                t_comm=rng.uniform(0.0, 2.0, K), f_mod=rng.uniform(0, 8e9, K), f_dat=rng.uniform(0, 8e9, K))


@pytest.mark.parametrize("seed", range(40))
def test_predict_matches_oracle(seed):
    d = _rand(seed)
    prof = Profile(d["m"], d["n"], d["dt"], d["phi"], list(d["t_gpu"]), list(d["t_comm"]), list(d["f_mod"]),
                   list(d["f_dat"]))
    rng = np.random.default_rng(1000 + seed)
    for _ in range(6):
        ms, ns = int(rng.integers(1, 128)), int(rng.integers(1, 9))
        o = o_predict(prof, ms, ns)
        per, it, pk = binding.predict(d["m"], d["n"], d["dt"], d["phi"], d["t_gpu"], d["t_comm"], d["f_mod"],
                                      d["f_dat"], ms, ns)
        for k in range(prof.K):
            for f in ("t_gpu", "t_com", "t_up", "t_down", "t_bub", "t_total", "mem"):
                assert per[k][f] == pytest.approx(o[f][k], rel=1e-12, abs=1e-300), (k, f)
        assert it == pytest.approx(o["iter_time"], rel=1e-12)
        assert pk == pytest.approx(o["peak_mem"], rel=1e-12)


@pytest.mark.parametrize("seed", range(30))
@pytest.mark.parametrize("objective", ["throughput", "time"])
def test_tune_matches_oracle(seed, objective):
    d = _rand(seed, S=50)
    prof = Profile(d["m"], d["n"], d["dt"], d["phi"], list(d["t_gpu"]), list(d["t_comm"]), list(d["f_mod"]),
                   list(d["f_dat"]))
    ms, ns = [1, 2, 4, 8, 16, 32, 64], [1, 2, 3, 4, 6, 8]
    mems = sorted(o_predict(prof, m, n)["peak_mem"] for m, n in itertools.product(ms, ns))
    for limit in (mems[0] * 0.5, mems[len(mems) // 3], mems[-1] * 2):
        o = o_tune(prof, ms, ns, limit, objective)
        b = binding.tune(d["m"], d["n"], d["dt"], d["phi"], d["t_gpu"], d["t_comm"], d["f_mod"], d["f_dat"], ms,
                         ns, limit, objective)
        if o is None:
            assert b is None
        else:
            assert (b[0], b[1]) == (o[0], o[1])
            assert b[2] == pytest.approx(o[2], rel=1e-12)


def test_predict_rejects_bad_profiles():
    d = _rand(0, K=2, S=4)
    bad_phi = np.array(d["phi"])
    bad_phi[0, 0] = 1.5
    with pytest.raises(binding.EAError):
        binding.predict(d["m"], d["n"], d["dt"], bad_phi, d["t_gpu"], d["t_comm"], d["f_mod"], d["f_dat"], 4, 1)
    with pytest.raises(binding.EAError):
        binding.predict(d["m"], d["n"], d["dt"], d["phi"], d["t_gpu"], d["t_comm"], d["f_mod"], d["f_dat"], 0, 1)
    with pytest.raises(binding.EAError):
        binding.predict(d["m"], d["n"], d["dt"], d["phi"], [-1.0, 1.0], d["t_comm"], d["f_mod"], d["f_dat"], 4, 1)
