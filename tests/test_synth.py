"""The seeded generator: host, element-wise and torch versions agree bit for bit."""
import numpy as np
import torch

import synth


def test_uniform_is_counter_based_and_bounded():
    a = synth.uniform((6, 7, 8), -1.0, 1.0, "k", 1)
    b = synth.uniform((6, 7, 8), -1.0, 1.0, "k", 1, chunk=5)
    assert np.array_equal(a, b)
    assert a.min() >= -1.0 and a.max() < 1.0
    assert not np.array_equal(a, synth.uniform((6, 7, 8), -1.0, 1.0, "k", 2))
    idx = np.array([0, 5, 100, 335])
    assert np.array_equal(synth.uniform_at(idx, -1.0, 1.0, "k", 1), a.ravel()[idx])


def test_uniform_torch_matches_numpy():
    a = synth.uniform((9, 10, 11), 0.5, 1.5, "t", "A")
    b = synth.uniform_torch((9, 10, 11), 0.5, 1.5, "t", "A", device="cpu", chunk=77)
    assert np.array_equal(a, b.numpy())
    if torch.cuda.is_available():  # pragma: no cover
        c = synth.uniform_torch((9, 10, 11), 0.5, 1.5, "t", "A", device="cuda")
        assert np.array_equal(a, c.cpu().numpy())
