"""Pins of oracle/nmi.py (NMI of [52]) against things other than itself."""
import math

import numpy as np
import pytest

from oracle.nmi import nmi


def test_identity_and_relabelling():
    rng = np.random.default_rng(0)
    x = rng.integers(0, 7, 200)
    perm = rng.permutation(7) + 100           # relabelled copy: same partition
    assert nmi(x, x) == pytest.approx(1.0, abs=1e-12)
    assert nmi(x, perm[x]) == pytest.approx(1.0, abs=1e-12)


def test_product_partition_is_zero():
    # X and Y independent by construction: every (a, b) cell has the same count -> I = 0
    x = np.repeat(np.arange(4), 6)            # 4 blocks of 6
    y = np.tile(np.arange(6), 4)              # crosses every block evenly
    assert nmi(x, y) == pytest.approx(0.0, abs=1e-12)


def test_hand_computed_example():
    # x = {0,1,2 | 3,4,5}, y = {0,1 | 2,3 | 4,5}; n = 6
    # n_ab: (0,0)=2 (0,1)=1 (1,1)=1 (1,2)=2;  n_a = 3,3;  n_b = 2,2,2
    # I = 2/6 ln(6*2/6) + 1/6 ln(6/6) + 1/6 ln(6/6) + 2/6 ln(6*2/6) = (2/3) ln 2
    # H(X) = ln 2, H(Y) = ln 3  ->  NMI = (2/3) ln 2 / sqrt(ln 2 ln 3)
    x = [0, 0, 0, 1, 1, 1]
    y = [0, 0, 1, 1, 2, 2]
    want = (2.0 / 3.0) * math.log(2) / math.sqrt(math.log(2) * math.log(3))
    assert nmi(x, y) == pytest.approx(want, rel=1e-14)
    assert nmi(y, x) == pytest.approx(want, rel=1e-14)


def test_degenerate_single_cluster():
    assert nmi([5] * 10, [1] * 10) == 1.0
    assert nmi([5] * 10, list(range(10))) == 0.0


def test_matches_sklearn_geometric():
    skm = pytest.importorskip("sklearn.metrics")
    rng = np.random.default_rng(1)
    for t in range(20):
        n = int(rng.integers(5, 500))
        x = rng.integers(0, int(rng.integers(1, 20)), n)
        y = np.where(rng.random(n) < 0.5, x, rng.integers(0, int(rng.integers(1, 20)), n))
        want = skm.normalized_mutual_info_score(x, y, average_method="geometric")
        assert nmi(x, y) == pytest.approx(want, abs=1e-10)
