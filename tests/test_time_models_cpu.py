"""tools/time_models.py (NEXT-4a, Fig. 10): the piecewise LR recovers exactly piecewise-
linear times (cross-validated RAE ~ 0) and the RAE matches its definition."""
import numpy as np

from tools import time_models as TM


def test_rae_definition():
    y = np.array([1.0, 2.0, 3.0, 4.0])
    assert TM.rae(y, y) == 0.0
    # mean 2.5: sum|mean - y| = 4; predicting the mean everywhere gives RAE 1
    assert TM.rae(np.full(4, 2.5), y) == 1.0
    assert abs(TM.rae(y + 0.4, y) - 1.6 / 4) < 1e-12


def test_piecewise_lr_exact_on_piecewise_linear_data():
    rng = np.random.default_rng(0)
    S = rng.uniform(20e6, 2000e6, 400)
    s = rng.uniform(0.2, 0.9, 400)
    beta = {b: (1e-5 * (b + 1), 2e-13 * (b + 2), -1e-13 * (b + 1)) for b in range(len(TM.BANDS))}
    t = np.array([beta[TM.band_of(si)][0] + beta[TM.band_of(si)][1] * Si + beta[TM.band_of(si)][2] * Si * si
                  for Si, si in zip(S, s)])
    X = np.stack([S, s], axis=1)
    assert TM.cv_rae(TM.PiecewiseLR, X, t) < 1e-6
