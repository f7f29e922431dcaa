"""bench.py host helpers (no GPU): the error ratio of Eq. 4."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_error_ratio_eq4():
    import bench
    gt = np.array([[1.0, 4.0, 9.0]])
    assert bench.error_ratio(gt, gt) == 1.0                              # exact answer: kappa = 1
    # kappa = mean of |v - N_i| / |v - I_i| = (1/1 + 2/3 + 3/3) / 3
    assert abs(bench.error_ratio(gt, np.array([[1.0, 9.0, 9.0]])) - (1 + 2 / 3 + 1) / 3) < 1e-12
    assert bench.error_ratio(gt, np.array([[1.0, 4.0, np.inf]])) == 2 / 3  # a padded slot contributes 0
    assert bench.error_ratio(np.array([[0.0]]), np.array([[0.0]])) == 1.0  # 0 / 0 (the query is a data point)
