"""Pins of the float64 oracle (oracle/ea_oracle.py) to things other than itself.

Each pin is a closed form, a library routine, an exact-rational hand
expansion or an invariant the paper states.  Together they fail on a dropped
term, a wrong sign, a wrong index or a swapped operand anywhere in the step
(see the mistake table in DESIGN.md "Oracle pins").

P1  alpha = 0  =>  N independent torch.optim.SGD(momentum, nesterov, wd) runs
    (north star; torch.optim is a library routine, float64 CPU).
P2  zero grads/momentum: sum_i x_i + x~ conserved when beta = N*alpha;
    D = mean(x) - x~ decays by (1 - alpha - beta); e_i = x_i - mean(x) by
    (1 - alpha) (north star: "shrink geometrically by the closed-form factor").
P3  paper mode (rho = 1) with x~_0 = mean(x_0): x~_t = mean_i x_i,t for any
    gradients ("stays the average").
P4  alpha = 1  =>  x_i,t+1 = x~_t + Delta_i (full dilution), Delta_i from
    torch.optim.SGD.
P5  N = 1, rho = 1, x_0 = x~_0  =>  one SGD trajectory and x~ == x.
P6  2 replicas x 8 params x 3 steps in exact rationals (fractions.Fraction),
    written as scalar EASGD-style formulas (north star "brute force").
P8  constant gradients with momentum, paper mode: closed forms for mean(x_t)
    and the gaps e_i,t.
P9  EASGD mode, plain SGD: the textbook synchronous EASGD recursion
    x~' = (1 - N*alpha) x~ + N*alpha * mean(x)  (Zhang et al., ref [35]).
"""
from fractions import Fraction

import numpy as np
import pytest
import torch

from oracle.ea_oracle import Hyper, ea_run, ea_step


def _rand_state(rng, n, p, spread=1e-3):
    x0 = rng.normal(0, 0.02, p)
    xs = [x0 + rng.normal(0, spread, p) for _ in range(n)]
    return xs, [np.zeros(p) for _ in range(n)], x0.copy()


def _grads(rng, n, p, steps, scale=1e-2):
    return [[rng.normal(0, scale, p) for _ in range(n)] for _ in range(steps)]


# ---------------------------------------------------------------- P1
@pytest.mark.parametrize("nesterov,wd", [(False, 0.0), (True, 0.0), (False, 1e-2), (True, 5e-3)])
@pytest.mark.parametrize("beta,rho", [(0.0, 1.0), (3.0, 0.0), (3.0, 1.0), (0.7, 0.3)])
def test_p1_alpha0_is_independent_torch_sgd(nesterov, wd, beta, rho):
    rng = np.random.default_rng(11)
    n, p, steps = 3, 257, 12
    lr, mu = 0.05, 0.9
    xs, ms, c = _rand_state(rng, n, p)
    gs = _grads(rng, n, p, steps)
    hp = Hyper(alpha=0.0, beta=beta, rho=rho, lr=lr, momentum=mu, weight_decay=wd, nesterov=nesterov)
    oxs, oms, _ = ea_run(xs, ms, c, gs, hp)
    for i in range(n):
        w = torch.nn.Parameter(torch.tensor(xs[i], dtype=torch.float64))
        opt = torch.optim.SGD([w], lr=lr, momentum=mu, weight_decay=wd, nesterov=nesterov)
        for t in range(steps):
            w.grad = torch.tensor(gs[t][i], dtype=torch.float64)
            opt.step()
        np.testing.assert_allclose(oxs[i], w.detach().numpy(), rtol=1e-13, atol=1e-16)
        np.testing.assert_allclose(oms[i], opt.state[w]["momentum_buffer"].numpy(), rtol=1e-13, atol=1e-16)


# ---------------------------------------------------------------- P2
@pytest.mark.parametrize("n,alpha", [(2, 0.5), (3, 1 / 3), (4, 0.1), (8, 0.125), (5, 0.03)])
@pytest.mark.parametrize("rho", [0.0, 1.0])
def test_p2_conservation_and_geometric_decay(n, alpha, rho):
    rng = np.random.default_rng(5)
    p, steps = 64, 25
    beta = n * alpha
    xs, ms, c = _rand_state(rng, n, p)
    c = c + rng.normal(0, 1e-3, p)          # D_0 != 0
    zero = [[np.zeros(p)] * n] * steps
    hp = Hyper(alpha=alpha, beta=beta, rho=rho, lr=0.05, momentum=0.9)
    total0 = sum(xs) + c
    d0 = np.mean(xs, axis=0) - c
    e0 = [x - np.mean(xs, axis=0) for x in xs]
    cur = (xs, ms, c)
    for t in range(1, steps + 1):
        cur = ea_step(*cur[:3], zero[t - 1], hp)
        x_t, _, c_t = cur
        np.testing.assert_allclose(sum(x_t) + c_t, total0, rtol=0, atol=1e-12)
        np.testing.assert_allclose(np.mean(x_t, axis=0) - c_t, (1 - alpha - beta) ** t * d0,
                                   rtol=1e-9, atol=1e-15)
        for i in range(n):
            np.testing.assert_allclose(x_t[i] - np.mean(x_t, axis=0), (1 - alpha) ** t * e0[i],
                                       rtol=1e-9, atol=1e-15)


@pytest.mark.parametrize("beta", [0.0, 0.25, 1.5])
def test_p2_gap_decay_any_beta(beta):
    """D_t = (1 - alpha - beta)^t D_0 holds for any beta (no conservation)."""
    rng = np.random.default_rng(6)
    n, p, alpha = 3, 40, 0.2
    xs, ms, c = _rand_state(rng, n, p)
    c = c + 0.01
    hp = Hyper(alpha=alpha, beta=beta, rho=1.0, lr=0.1, momentum=0.5)
    d0 = np.mean(xs, axis=0) - c
    x_t, _, c_t = ea_run(xs, ms, c, [[np.zeros(p)] * n] * 7, hp)
    np.testing.assert_allclose(np.mean(x_t, axis=0) - c_t, (1 - alpha - beta) ** 7 * d0, rtol=1e-10)


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("beta", [0.0, 1.0, 1.5])   # |1-alpha-beta| <= 1: rounding in D does not grow
@pytest.mark.parametrize("nesterov,wd", [(False, 0.0), (True, 1e-3)])
def test_p3_center_stays_the_average(beta, nesterov, wd):
    rng = np.random.default_rng(7)
    n, p, steps = 3, 300, 50
    xs, ms, _ = _rand_state(rng, n, p)
    c = np.mean(xs, axis=0)
    hp = Hyper(alpha=1 / n, beta=beta, rho=1.0, lr=0.05, momentum=0.9, weight_decay=wd, nesterov=nesterov)
    cur = (xs, ms, c)
    for g in _grads(rng, n, p, steps):
        cur = ea_step(*cur, g, hp)
        np.testing.assert_allclose(cur[2], np.mean(cur[0], axis=0), rtol=0, atol=1e-15)


# ---------------------------------------------------------------- P4
def test_p4_alpha1_full_dilution():
    rng = np.random.default_rng(8)
    n, p, lr, mu = 4, 100, 0.05, 0.9
    xs, ms, c = _rand_state(rng, n, p)
    ms = [rng.normal(0, 1e-2, p) for _ in range(n)]
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=1.0, beta=0.3, rho=1.0, lr=lr, momentum=mu)
    nx, _, _ = ea_step(xs, ms, c, g, hp)
    for i in range(n):
        w = torch.nn.Parameter(torch.tensor(xs[i], dtype=torch.float64))
        opt = torch.optim.SGD([w], lr=lr, momentum=mu)
        opt.state[w]["momentum_buffer"] = torch.tensor(ms[i], dtype=torch.float64)
        w.grad = torch.tensor(g[i], dtype=torch.float64)
        before = w.detach().clone()
        opt.step()
        delta = (w.detach() - before).numpy()
        np.testing.assert_allclose(nx[i], c + delta, rtol=1e-12, atol=1e-17)


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (0.3, 0.7), (0.0, 2.0)])
def test_p5_single_pipeline_is_sgd(alpha, beta):
    rng = np.random.default_rng(9)
    p, steps, lr, mu = 50, 20, 0.05, 0.9
    x0 = rng.normal(0, 0.02, p)
    gs = _grads(rng, 1, p, steps)
    xs, ms, c = ea_run([x0], [np.zeros(p)], x0, gs, Hyper(alpha=alpha, beta=beta, rho=1.0, lr=lr, momentum=mu))
    w = torch.nn.Parameter(torch.tensor(x0, dtype=torch.float64))
    opt = torch.optim.SGD([w], lr=lr, momentum=mu)
    for t in range(steps):
        w.grad = torch.tensor(gs[t][0], dtype=torch.float64)
        opt.step()
    np.testing.assert_allclose(xs[0], w.detach().numpy(), rtol=1e-13, atol=1e-17)
    np.testing.assert_allclose(c, xs[0], rtol=1e-13, atol=1e-17)


# ---------------------------------------------------------------- P6
def _brute_force_fraction(x, m, c, g, alpha, beta, rho, lr, mu):
    """Hand expansion, element by element, in the EASGD 'elastic force' form
    x' = x - lr*m' - alpha*(x - c) (algebraically the paper's (1-a):a dilution
    plus local update), center c' = c + (rho*sum(Delta) + beta*sum(x - c)) / N."""
    N = len(x)
    P = len(c)
    nx = [[None] * P for _ in range(N)]
    nm = [[None] * P for _ in range(N)]
    nc = [None] * P
    for j in range(P):
        sum_delta = Fraction(0)
        sum_gap = Fraction(0)
        for i in range(N):
            m_new = mu * m[i][j] + g[i][j]
            delta = -lr * m_new
            nm[i][j] = m_new
            nx[i][j] = x[i][j] - lr * m_new - alpha * (x[i][j] - c[j])
            sum_delta += delta
            sum_gap += x[i][j] - c[j]
        nc[j] = c[j] + (rho * sum_delta + beta * sum_gap) / N
    return nx, nm, nc


@pytest.mark.parametrize("alpha,beta,rho", [(Fraction(1, 2), Fraction(0), Fraction(1)),
                                            (Fraction(1, 2), Fraction(1), Fraction(0)),
                                            (Fraction(1, 3), Fraction(2, 3), Fraction(1))])
def test_p6_brute_force_fractions(alpha, beta, rho):
    rng = np.random.default_rng(10)
    N, P, steps = 2, 8, 3
    lr, mu = Fraction(1, 20), Fraction(9, 10)
    to_fr = lambda a: [Fraction(int(v), 1 << 20) for v in a]   # exact dyadic inputs
    x = [to_fr(rng.integers(-20000, 20000, P)) for _ in range(N)]
    c = to_fr(rng.integers(-20000, 20000, P))
    m = [[Fraction(0)] * P for _ in range(N)]
    gs = [[to_fr(rng.integers(-10000, 10000, P)) for _ in range(N)] for _ in range(steps)]
    fx, fm, fc = x, m, c
    for t in range(steps):
        fx, fm, fc = _brute_force_fraction(fx, fm, fc, gs[t], alpha, beta, rho, lr, mu)
    hp = Hyper(alpha=float(alpha), beta=float(beta), rho=float(rho), lr=float(lr), momentum=float(mu))
    f = lambda a: np.array([float(v) for v in a])
    ox, om, oc = ea_run([f(v) for v in x], [np.zeros(P)] * N, f(c),
                        [[f(v) for v in gs[t]] for t in range(steps)], hp)
    for i in range(N):
        np.testing.assert_allclose(ox[i], f(fx[i]), rtol=1e-14, atol=1e-17)
        np.testing.assert_allclose(om[i], f(fm[i]), rtol=1e-14, atol=1e-17)
    np.testing.assert_allclose(oc, f(fc), rtol=1e-14, atol=1e-17)


# ---------------------------------------------------------------- P8
def test_p8_constant_gradient_closed_form():
    rng = np.random.default_rng(12)
    n, p, steps, alpha, lr, mu = 3, 20, 15, 0.25, 0.05, 0.9
    xs, ms, _ = _rand_state(rng, n, p)
    c = np.mean(xs, axis=0)
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=alpha, beta=0.0, rho=1.0, lr=lr, momentum=mu)
    ox, _, oc = ea_run(xs, ms, c, [g] * steps, hp)
    # momentum after s+1 updates with constant g: g * (1 - mu^(s+1)) / (1 - mu)
    delta = lambda i, s: -lr * g[i] * (1 - mu ** (s + 1)) / (1 - mu)
    mean_delta = lambda s: sum(delta(i, s) for i in range(n)) / n
    mean_x = np.mean(xs, axis=0) + sum(mean_delta(s) for s in range(steps))
    np.testing.assert_allclose(np.mean(ox, axis=0), mean_x, rtol=1e-12, atol=1e-16)
    np.testing.assert_allclose(oc, mean_x, rtol=1e-12, atol=1e-16)
    for i in range(n):
        e0 = xs[i] - np.mean(xs, axis=0)
        e_t = (1 - alpha) ** steps * e0 + sum((1 - alpha) ** (steps - 1 - s) * (delta(i, s) - mean_delta(s))
                                             for s in range(steps))
        np.testing.assert_allclose(ox[i] - np.mean(ox, axis=0), e_t, rtol=1e-10, atol=1e-16)


# ---------------------------------------------------------------- P9
def test_p9_textbook_synchronous_easgd():
    rng = np.random.default_rng(13)
    n, p, steps, alpha, lr = 4, 33, 10, 0.1, 0.05
    xs, ms, c = _rand_state(rng, n, p)
    gs = _grads(rng, n, p, steps)
    ox, _, oc = ea_run(xs, ms, c, gs, Hyper(alpha=alpha, beta=n * alpha, rho=0.0, lr=lr, momentum=0.0))
    ex, ec = [x.copy() for x in xs], c.copy()
    for t in range(steps):
        new_c = (1 - n * alpha) * ec + n * alpha * np.mean(ex, axis=0)
        ex = [ex[i] - lr * gs[t][i] - alpha * (ex[i] - ec) for i in range(n)]
        ec = new_c
    for i in range(n):
        np.testing.assert_allclose(ox[i], ex[i], rtol=1e-12, atol=1e-17)
    np.testing.assert_allclose(oc, ec, rtol=1e-12, atol=1e-17)


# ---------------------------------------------------------------- structure
def test_replica_permutation_equivariance():
    rng = np.random.default_rng(14)
    n, p = 4, 30
    xs, _, c = _rand_state(rng, n, p)
    ms = [rng.normal(0, 1e-2, p) for _ in range(n)]
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=0.3, beta=0.5, rho=1.0, lr=0.05, momentum=0.9, nesterov=True)
    a = ea_step(xs, ms, c, g, hp)
    perm = [2, 0, 3, 1]
    b = ea_step([xs[k] for k in perm], [ms[k] for k in perm], c, [g[k] for k in perm], hp)
    for pos, k in enumerate(perm):
        np.testing.assert_allclose(b[0][pos], a[0][k], rtol=1e-15)
        np.testing.assert_allclose(b[1][pos], a[1][k], rtol=1e-15)
    np.testing.assert_allclose(b[2], a[2], rtol=1e-14)


def test_inputs_not_modified_and_fixed_point():
    p, n = 16, 3
    x = np.linspace(-1, 1, p)
    xs, ms, c = [x.copy() for _ in range(n)], [np.zeros(p)] * n, x.copy()
    hp = Hyper(alpha=0.5, beta=1.5, rho=1.0, lr=0.1, momentum=0.9)
    nx, nm, nc = ea_step(xs, ms, c, [np.zeros(p)] * n, hp)
    for i in range(n):
        np.testing.assert_array_equal(nx[i], x)
        np.testing.assert_array_equal(xs[i], x)
    np.testing.assert_array_equal(nc, x)


# ---------------------------------------------------------------- Adam / AdamW (row f1, reading c21)
from oracle.ea_oracle import ea_step_adam  # noqa: E402


@pytest.mark.parametrize("decoupled,wd", [(False, 0.0), (False, 1e-2), (True, 1e-2), (True, 0.0)])
@pytest.mark.parametrize("beta,rho", [(0.0, 1.0), (2.0, 0.0)])
def test_p1_adam_alpha0_is_independent_torch_adam(decoupled, wd, beta, rho):
    """alpha = 0 => N independent torch.optim.Adam / AdamW trajectories (library routine)."""
    rng = np.random.default_rng(21)
    n, p, steps, lr = 2, 300, 15, 1e-3
    xs, _, c = _rand_state(rng, n, p)
    gs = _grads(rng, n, p, steps)
    hp = Hyper(alpha=0.0, beta=beta, rho=rho, lr=lr, weight_decay=wd, beta1=0.9, beta2=0.999, eps=1e-8)
    ox = [x.copy() for x in xs]
    om = [np.zeros(p) for _ in range(n)]
    ov = [np.zeros(p) for _ in range(n)]
    oc = c.copy()
    for t in range(steps):
        ox, om, ov, oc = ea_step_adam(ox, om, ov, oc, gs[t], hp, t + 1, decoupled)
    for i in range(n):
        w = torch.nn.Parameter(torch.tensor(xs[i], dtype=torch.float64))
        cls = torch.optim.AdamW if decoupled else torch.optim.Adam
        opt = cls([w], lr=lr, betas=(0.9, 0.999), eps=1e-8, weight_decay=wd)
        for t in range(steps):
            w.grad = torch.tensor(gs[t][i], dtype=torch.float64)
            opt.step()
        np.testing.assert_allclose(ox[i], w.detach().numpy(), rtol=1e-12, atol=1e-16)
        np.testing.assert_allclose(om[i], opt.state[w]["exp_avg"].numpy(), rtol=1e-12, atol=1e-18)
        np.testing.assert_allclose(ov[i], opt.state[w]["exp_avg_sq"].numpy(), rtol=1e-12, atol=1e-20)


@pytest.mark.parametrize("decoupled", [False, True])
def test_p3_adam_center_stays_the_average(decoupled):
    """'stays the average' holds whatever the optimizer (rho = 1)."""
    rng = np.random.default_rng(22)
    n, p = 3, 200
    xs, _, _ = _rand_state(rng, n, p)
    c = np.mean(xs, axis=0)
    hp = Hyper(alpha=1 / n, beta=0.5, rho=1.0, lr=1e-3, weight_decay=1e-2)
    ms = [np.zeros(p)] * n
    vs = [np.zeros(p)] * n
    for t, g in enumerate(_grads(rng, n, p, 30)):
        xs, ms, vs, c = ea_step_adam(xs, ms, vs, c, g, hp, t + 1, decoupled)
        np.testing.assert_allclose(c, np.mean(xs, axis=0), rtol=0, atol=1e-15)


def test_p2_adam_zero_gradients_decay():
    """Zero gradients and zero moments: Delta = 0, so the P2 closed forms hold for Adam too."""
    rng = np.random.default_rng(23)
    n, p, alpha = 4, 50, 0.1
    xs, _, c = _rand_state(rng, n, p)
    c = c + 1e-3
    hp = Hyper(alpha=alpha, beta=n * alpha, rho=1.0, lr=1e-3)
    d0 = np.mean(xs, axis=0) - c
    total0 = sum(xs) + c
    ms = [np.zeros(p)] * n
    vs = [np.zeros(p)] * n
    for t in range(10):
        xs, ms, vs, c = ea_step_adam(xs, ms, vs, c, [np.zeros(p)] * n, hp, t + 1)
    np.testing.assert_allclose(np.mean(xs, axis=0) - c, (1 - alpha - n * alpha) ** 10 * d0, rtol=1e-9, atol=1e-16)
    np.testing.assert_allclose(sum(xs) + c, total0, rtol=0, atol=1e-13)


# ---------------------------------------------------------------- stale center (row f4, reading c28)
from oracle.ea_oracle import ea_step_stale  # noqa: E402


def test_stale_with_equal_centers_is_the_synchronous_step():
    rng = np.random.default_rng(31)
    n, p = 3, 100
    xs, _, c = _rand_state(rng, n, p)
    ms = [rng.normal(0, 1e-2, p) for _ in range(n)]
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=0.3, beta=0.9, rho=1.0, lr=0.05, momentum=0.9)
    a = ea_step(xs, ms, c, g, hp)
    b = ea_step_stale(xs, ms, c, c, g, hp)
    for i in range(n):
        np.testing.assert_array_equal(a[0][i], b[0][i])
    np.testing.assert_array_equal(a[2], b[2])
    np.testing.assert_array_equal(b[3], c)


@pytest.mark.parametrize("n,alpha,rho", [(2, 0.5, 1.0), (3, 0.2, 0.0), (4, 0.1, 1.0)])
def test_stale_zero_gradient_state_space_closed_form(n, alpha, rho):
    """Zero gradients/momentum: (mean x_{t+1}, x~_{t+1}, x~_t) = A (mean x_t, x~_t, x~_{t-1}) with
    A = [[1-a, 0, a], [b, 1, -b], [0, 1, 0]]  (beta = b), so the trajectory is a matrix power;
    Sum x + x~ is conserved when beta = N alpha; deviations e_i decay by (1 - alpha)."""
    rng = np.random.default_rng(32)
    p, steps = 50, 12
    beta = n * alpha
    xs, ms, c = _rand_state(rng, n, p)
    c = c + rng.normal(0, 1e-3, p)
    hp = Hyper(alpha=alpha, beta=beta, rho=rho, lr=0.05, momentum=0.9)
    A = np.array([[1 - alpha, 0.0, alpha], [beta, 1.0, -beta], [0.0, 1.0, 0.0]])
    s0 = np.stack([np.mean(xs, axis=0), c, c])                 # x~_{-1} := x~_0
    e0 = [x - np.mean(xs, axis=0) for x in xs]
    total0 = sum(xs) + c
    cur_x, cur_m, cur_c, prev_c = xs, ms, c, c
    for t in range(1, steps + 1):
        cur_x, cur_m, cur_c, prev_c = ea_step_stale(cur_x, cur_m, cur_c, prev_c, [np.zeros(p)] * n, hp)
        st = np.linalg.matrix_power(A, t) @ s0
        np.testing.assert_allclose(np.mean(cur_x, axis=0), st[0], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(cur_c, st[1], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(prev_c, st[2], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(sum(cur_x) + cur_c, total0, rtol=0, atol=1e-12)
        for i in range(n):
            np.testing.assert_allclose(cur_x[i] - np.mean(cur_x, axis=0), (1 - alpha) ** t * e0[i], rtol=1e-9,
                                       atol=1e-15)


# ---------------------------------------------------------------- stale center with Adam / AdamW (f4 + f1)
from oracle.ea_oracle import ea_step_adam_stale  # noqa: E402


@pytest.mark.parametrize("decoupled", [False, True])
def test_adam_stale_with_equal_centers_is_the_synchronous_adam_step(decoupled):
    rng = np.random.default_rng(33)
    n, p = 3, 100
    xs, _, c = _rand_state(rng, n, p)
    ms = [rng.normal(0, 1e-3, p) for _ in range(n)]
    vs = [rng.uniform(0, 1e-4, p) for _ in range(n)]
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=0.3, beta=0.9, rho=1.0, lr=1e-3, weight_decay=1e-2)
    a = ea_step_adam(xs, ms, vs, c, g, hp, 4, decoupled=decoupled)
    b = ea_step_adam_stale(xs, ms, vs, c, c, g, hp, 4, decoupled=decoupled)
    for i in range(n):
        np.testing.assert_array_equal(a[0][i], b[0][i])
        np.testing.assert_array_equal(a[1][i], b[1][i])
        np.testing.assert_array_equal(a[2][i], b[2][i])
    np.testing.assert_array_equal(a[3], b[3])
    np.testing.assert_array_equal(b[4], c)


def test_adam_stale_alpha0_is_independent_torch_adam():
    """alpha = 0: the stale reference never feeds back, so every replica is torch.optim.Adam (float64)."""
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(34)
    n, p, steps = 2, 40, 6
    xs, _, c = _rand_state(rng, n, p)
    hp = Hyper(alpha=0.0, beta=0.7, rho=1.0, lr=1e-2, weight_decay=1e-2)
    grads = [[rng.normal(0, 1e-2, p) for _ in range(n)] for _ in range(steps)]
    ref = []
    for i in range(n):
        w = torch.tensor(xs[i], dtype=torch.float64, requires_grad=True)
        opt = torch.optim.Adam([w], lr=hp.lr, betas=(hp.beta1, hp.beta2), eps=hp.eps, weight_decay=hp.weight_decay)
        for t in range(steps):
            w.grad = torch.tensor(grads[t][i], dtype=torch.float64)
            opt.step()
        ref.append(w.detach().numpy())
    cur = (xs, [np.zeros(p)] * n, [np.zeros(p)] * n, c, c)
    for t in range(steps):
        x_, m_, v_, c_new, c_old = ea_step_adam_stale(cur[0], cur[1], cur[2], cur[3], cur[4], grads[t], hp, t + 1)
        cur = (x_, m_, v_, c_new, c_old)
    for i in range(n):
        np.testing.assert_allclose(cur[0][i], ref[i], rtol=1e-13, atol=1e-15)


@pytest.mark.parametrize("n,alpha,rho", [(2, 0.5, 1.0), (3, 0.2, 0.0)])
def test_adam_stale_zero_gradient_state_space_closed_form(n, alpha, rho):
    """Zero gradients and moments give Delta = 0 under Adam too, so the stale state-space closed form
    (mean x, x~_t, x~_{t-1}) = A^t s_0 holds with A = [[1-a, 0, a], [b, 1, -b], [0, 1, 0]]."""
    rng = np.random.default_rng(35)
    p, steps = 50, 10
    beta = n * alpha
    xs, _, c = _rand_state(rng, n, p)
    c = c + rng.normal(0, 1e-3, p)
    hp = Hyper(alpha=alpha, beta=beta, rho=rho, lr=1e-3)
    A = np.array([[1 - alpha, 0.0, alpha], [beta, 1.0, -beta], [0.0, 1.0, 0.0]])
    s0 = np.stack([np.mean(xs, axis=0), c, c])
    total0 = sum(xs) + c
    z = [np.zeros(p)] * n
    cur_x, cur_m, cur_v, cur_c, prev_c = xs, z, z, c, c
    for t in range(1, steps + 1):
        cur_x, cur_m, cur_v, cur_c, prev_c = ea_step_adam_stale(cur_x, cur_m, cur_v, cur_c, prev_c, z, hp, t)
        st = np.linalg.matrix_power(A, t) @ s0
        np.testing.assert_allclose(np.mean(cur_x, axis=0), st[0], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(cur_c, st[1], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(prev_c, st[2], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(sum(cur_x) + cur_c, total0, rtol=0, atol=1e-12)


# ---------------------------------------------------------------- ASGD (row f1, reading c29)
@pytest.mark.parametrize("wd,lambd,t0", [(0.0, 1e-4, 1e6), (1e-2, 5e-2, 3.0), (0.0, 2e-1, 0.0)])
@pytest.mark.parametrize("beta,rho", [(0.0, 1.0), (2.0, 0.0), (0.7, 0.3)])
def test_p1_asgd_alpha0_is_independent_torch_asgd(wd, lambd, t0, beta, rho):
    """alpha = 0 => N independent torch.optim.ASGD trajectories, iterate AND average ax
    (library routine; t0 small so the running average with mu < 1 is exercised)."""
    from oracle.ea_oracle import ea_step_asgd
    rng = np.random.default_rng(31)
    n, p, steps, lr, a = 3, 211, 14, 0.5, 0.75
    xs, _, c = _rand_state(rng, n, p)
    gs = _grads(rng, n, p, steps)
    hp = Hyper(alpha=0.0, beta=beta, rho=rho, lr=lr, weight_decay=wd, asgd_lambd=lambd, asgd_alpha=a, asgd_t0=t0)
    ox, oa, oc = [x.copy() for x in xs], [np.zeros(p) for _ in range(n)], c.copy()
    for t in range(steps):
        ox, oa, oc = ea_step_asgd(ox, oa, oc, gs[t], hp, t + 1)
    # torch keeps ASGD's eta and mu as scalar tensors of the default dtype: float64 here, so the library
    # routine runs entirely in float64 like the oracle
    prev = torch.get_default_dtype()
    torch.set_default_dtype(torch.float64)
    try:
        for i in range(n):
            w = torch.nn.Parameter(torch.tensor(xs[i], dtype=torch.float64))
            opt = torch.optim.ASGD([w], lr=lr, lambd=lambd, alpha=a, t0=t0, weight_decay=wd)
            for t in range(steps):
                w.grad = torch.tensor(gs[t][i], dtype=torch.float64)
                opt.step()
            np.testing.assert_allclose(ox[i], w.detach().numpy(), rtol=1e-13, atol=1e-16)
            np.testing.assert_allclose(oa[i], opt.state[w]["ax"].numpy(), rtol=1e-13, atol=1e-16)
    finally:
        torch.set_default_dtype(prev)


def test_asgd_average_is_the_mean_of_the_iterates():
    """t0 = 0: mu_t = 1/max(1, t-1), so after t >= 2 steps the average is the arithmetic mean of the
    optimizer's iterates x_2 .. x_t (the definition of averaged SGD, ref [27]), computed here from the
    replica trajectory itself (alpha = 0)."""
    from oracle.ea_oracle import ea_step_asgd
    rng = np.random.default_rng(32)
    n, p, steps = 2, 64, 9
    xs, _, c = _rand_state(rng, n, p)
    hp = Hyper(alpha=0.0, beta=0.0, rho=1.0, lr=0.3, asgd_lambd=1e-2, asgd_t0=0.0)
    traj = [[] for _ in range(n)]
    axs = [np.zeros(p) for _ in range(n)]
    for t, g in enumerate(_grads(rng, n, p, steps)):
        xs, axs, c = ea_step_asgd(xs, axs, c, g, hp, t + 1)
        for i in range(n):
            traj[i].append(xs[i])
    for i in range(n):
        np.testing.assert_allclose(axs[i], np.mean(traj[i][1:], axis=0), rtol=1e-13, atol=1e-17)


def test_asgd_zero_gradients_closed_form():
    """Zero gradients, N = 1, alpha = 0: x_t = x_0 * prod_k (1 - lambd*eta_k) with
    eta_k = lr / (1 + lambd*lr*(k-1))**a -- the decay term alone, hand-evaluated."""
    from oracle.ea_oracle import ea_step_asgd
    rng = np.random.default_rng(33)
    p, steps, lr, lambd, a = 50, 12, 0.4, 0.1, 0.75
    x0 = rng.normal(0, 0.02, p)
    hp = Hyper(alpha=0.0, beta=0.0, rho=1.0, lr=lr, asgd_lambd=lambd, asgd_alpha=a)
    xs, axs, c = [x0.copy()], [np.zeros(p)], x0.copy()
    f = 1.0
    for k in range(1, steps + 1):
        xs, axs, c = ea_step_asgd(xs, axs, c, [np.zeros(p)], hp, k)
        f *= 1.0 - lambd * lr / (1.0 + lambd * lr * (k - 1)) ** a
        np.testing.assert_allclose(xs[0], x0 * f, rtol=1e-14, atol=0)
        np.testing.assert_allclose(c, x0 * f, rtol=1e-14, atol=0)   # N = 1, rho = 1: x~ follows x


def test_p3_asgd_center_stays_the_average():
    """'stays the average' with ASGD as the local optimizer (rho = 1, centered init)."""
    from oracle.ea_oracle import ea_step_asgd
    rng = np.random.default_rng(34)
    n, p = 4, 150
    xs, _, _ = _rand_state(rng, n, p)
    c = np.mean(xs, axis=0)
    hp = Hyper(alpha=1 / n, beta=0.4, rho=1.0, lr=0.2, weight_decay=1e-3, asgd_lambd=1e-2, asgd_t0=2.0)
    axs = [np.zeros(p)] * n
    for t, g in enumerate(_grads(rng, n, p, 20)):
        xs, axs, c = ea_step_asgd(xs, axs, c, g, hp, t + 1)
        np.testing.assert_allclose(c, np.mean(xs, axis=0), rtol=0, atol=1e-15)


# ---------------------------------------------------------------- stale center with ASGD (rows f1 x f4)
def test_asgd_stale_with_equal_centers_is_the_synchronous_asgd_step():
    from oracle.ea_oracle import ea_step_asgd, ea_step_asgd_stale
    rng = np.random.default_rng(36)
    n, p = 3, 100
    xs, _, c = _rand_state(rng, n, p)
    axs = [x + rng.normal(0, 1e-4, p) for x in xs]
    g = [rng.normal(0, 1e-2, p) for _ in range(n)]
    hp = Hyper(alpha=0.3, beta=0.9, rho=1.0, lr=0.2, weight_decay=1e-3, asgd_lambd=1e-2, asgd_t0=1.0)
    a = ea_step_asgd(xs, axs, c, g, hp, 5)
    b = ea_step_asgd_stale(xs, axs, c, c, g, hp, 5)
    for i in range(n):
        np.testing.assert_array_equal(a[0][i], b[0][i])
        np.testing.assert_array_equal(a[1][i], b[1][i])
    np.testing.assert_array_equal(a[2], b[2])
    np.testing.assert_array_equal(b[3], c)


def test_asgd_stale_alpha0_is_independent_torch_asgd():
    """alpha = 0: the (stale) center never feeds back, so each replica is torch.optim.ASGD (float64)."""
    from oracle.ea_oracle import ea_step_asgd_stale
    rng = np.random.default_rng(37)
    n, p, steps, lr = 2, 120, 10, 0.3
    xs, _, c = _rand_state(rng, n, p)
    gs = _grads(rng, n, p, steps)
    hp = Hyper(alpha=0.0, beta=1.0, rho=1.0, lr=lr, weight_decay=1e-3, asgd_lambd=5e-2, asgd_t0=2.0)
    ox, oa, oc, op = [x.copy() for x in xs], [np.zeros(p) for _ in range(n)], c.copy(), c.copy()
    for t in range(steps):
        ox, oa, oc, op = ea_step_asgd_stale(ox, oa, oc, op, gs[t], hp, t + 1)
    prev = torch.get_default_dtype()
    torch.set_default_dtype(torch.float64)
    try:
        for i in range(n):
            w = torch.nn.Parameter(torch.tensor(xs[i], dtype=torch.float64))
            opt = torch.optim.ASGD([w], lr=lr, lambd=5e-2, alpha=0.75, t0=2.0, weight_decay=1e-3)
            for t in range(steps):
                w.grad = torch.tensor(gs[t][i], dtype=torch.float64)
                opt.step()
            np.testing.assert_allclose(ox[i], w.detach().numpy(), rtol=1e-13, atol=1e-16)
            np.testing.assert_allclose(oa[i], opt.state[w]["ax"].numpy(), rtol=1e-13, atol=1e-16)
    finally:
        torch.set_default_dtype(prev)


@pytest.mark.parametrize("n,alpha,rho", [(2, 0.5, 1.0), (4, 0.25, 0.0), (3, 0.1, 1.0)])
def test_asgd_stale_zero_gradient_state_space_closed_form(n, alpha, rho):
    """Zero gradients and no decay term (lambd = 0) give Delta = 0, so the stale state-space closed form
    (mean x, x~_t, x~_{t-1}) = A^t s_0 with A = [[1-a, 0, a], [b, 1, -b], [0, 1, 0]] holds with ASGD too."""
    from oracle.ea_oracle import ea_step_asgd_stale
    rng = np.random.default_rng(38)
    p, steps = 50, 10
    beta = n * alpha
    xs, _, c = _rand_state(rng, n, p)
    c = c + rng.normal(0, 1e-3, p)
    hp = Hyper(alpha=alpha, beta=beta, rho=rho, lr=0.1, asgd_lambd=0.0, asgd_t0=0.0)
    A = np.array([[1 - alpha, 0.0, alpha], [beta, 1.0, -beta], [0.0, 1.0, 0.0]])
    s0 = np.stack([np.mean(xs, axis=0), c, c])
    z = [np.zeros(p)] * n
    cur_x, cur_a, cur_c, prev_c = xs, z, c, c
    for t in range(1, steps + 1):
        cur_x, cur_a, cur_c, prev_c = ea_step_asgd_stale(cur_x, cur_a, cur_c, prev_c, z, hp, t)
        st = np.linalg.matrix_power(A, t) @ s0
        np.testing.assert_allclose(np.mean(cur_x, axis=0), st[0], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(cur_c, st[1], rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(prev_c, st[2], rtol=1e-12, atol=1e-15)
