"""The shared input generators are deterministic and backend-independent."""
import numpy as np
import torch

from inputs import counter_u64_np, counter_u64_torch, powerlaw_edges, rmat_edges_np, rmat_edges_torch
from inputs.graphs import WORKLOADS


def test_counter_rng_numpy_equals_torch():
    a = counter_u64_np(123, 7, 1000, 5000)
    b = counter_u64_torch(123, 7, 1000, 5000).numpy().view(np.uint64)
    assert np.array_equal(a, b)
    # known-answer: splitmix64 of state GOLDEN*1 with seed key 0 is stable
    assert counter_u64_np(0, 0, 0, 1)[0] == counter_u64_np(0, 0, 0, 2)[0]


def test_rmat_numpy_equals_torch():
    e_np = rmat_edges_np(10, 8, seed=3)
    e_t = rmat_edges_torch(10, 8, seed=3, chunk=1000).numpy().astype(np.int64)
    assert np.array_equal(e_np, e_t)
    assert e_np.min() >= 0 and e_np.max() < 1 << 10
    # skew: the a-quadrant dominates, vertex 0 is the heaviest
    deg = np.bincount(e_np.ravel(), minlength=1 << 10)
    assert deg.argmax() == 0


def test_powerlaw_exact_unique_edges():
    p = WORKLOADS["pl2k"][1]
    e = powerlaw_edges(**p)
    assert e.shape == (p["m"], 2)
    assert (e[:, 0] < e[:, 1]).all()
    keys = e[:, 0] * p["n"] + e[:, 1]
    assert np.unique(keys).size == p["m"]
    assert np.array_equal(e, powerlaw_edges(**p))  # reproducible


def test_internet_like_shape():
    p = WORKLOADS["internet"][1]
    e = powerlaw_edges(**p)
    deg = np.bincount(e.ravel(), minlength=p["n"])
    assert e.shape[0] == 193620
    assert 100 <= deg.max() <= 200          # Table 1 "internet": d_max 151
    assert abs(2 * 193620 / 124651 - 3.1) < 0.05
