"""The seeded input generators (no method arithmetic): shapes, determinism, phantom values."""
import numpy as np

from paper_conf_sc_hidayetoglubgrg19_b200 import inputs


def test_phantom_values():
    n = 64
    x = inputs.shepp_logan(n).reshape(n, n)
    # centre of the modified Shepp-Logan phantom: 1.0 - 0.8 = 0.2 (ellipses 1 and 2 only)
    assert abs(x[n // 2, n // 2] - 0.2) < 1e-12
    # corners are outside every ellipse
    assert x[0, 0] == 0.0 and x[-1, -1] == 0.0
    assert x.min() >= -1e-12 and x.max() <= 1.0 + 1e-12


def test_seeded_vectors_deterministic():
    a = inputs.uniform(1000, inputs.seed_for(3))
    b = inputs.uniform(1000, inputs.seed_for(3))
    assert np.array_equal(a, b) and a.dtype == np.float32
    assert 0.0 <= a.min() and a.max() < 1.0
    assert inputs.CONFIGS[3] == (1024, 1500, 1024)
