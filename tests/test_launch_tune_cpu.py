"""The Alg. 1 engine of tools/launch_tune.py (§IV-D) on CPU: the GP interpolates its
samples, and BO (s1 = 10, s2 = 25) finds the minimum of a smooth synthetic objective over a
(grid, variant) space of the kernel's shape in 35 evaluations, at least as well as 35 random ones."""
import numpy as np

from tools import launch_tune as LT


def test_gp_interpolates():
    X = np.linspace(0, 1, 8)[:, None]
    y = np.sin(3 * X[:, 0])
    mu, sd = LT.GP(noise=1e-8).fit(X, y).predict(X)
    assert np.max(np.abs(mu - y)) < 1e-3 and np.all(sd < 1e-2)


def test_bayes_opt_finds_minimum():
    space = [(q, v) for v in range(4) for q in range(1, 297)]

    def f(p):  # a Fig. 5-like bowl: time falls with the grid, then rises; variant 2 is best
        q, v = p
        return 44.0 * (1 + 0.5 * abs(v - 2)) * (1 + (np.log(q) - np.log(197)) ** 2)

    (bp, by), D = LT.bayes_opt(space, f, s1=10, s2=25, seed=3)
    assert len(D) == 35 and len({p for p, _ in D}) == 35
    best = min(f(p) for p in space)
    assert by <= best * 1.05
    rng = np.random.default_rng(1)
    rnd = min(f(space[i]) for i in rng.choice(len(space), 35, replace=False))
    assert by <= rnd
