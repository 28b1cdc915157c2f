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


def test_recipes_match_the_input_builders():
    """bench.py builds BASELINE inputs on the device from synth.recipe(); they
    are bit-identical to the *_inputs() arrays the parity tests use."""
    dims = (5, 6, 7)
    builders = {"jacobi7": synth.jacobi7_inputs, "lap25": synth.lap25_inputs, "smooth27": synth.smooth27_inputs,
                "hypterm": synth.hypterm_inputs, "rhs4center": synth.rhs4_inputs}
    for name, fn in builders.items():
        cfg, a3, a1, sc = synth.recipe(name)
        ins, sc_ref = fn(dims, cfg=cfg)
        assert sc == sc_ref, name
        assert set(ins) == set(a3) | set(a1), name
        for k, (lo, hi) in a3.items():
            t = synth.uniform_torch(dims, lo, hi, cfg, k, device="cpu")
            assert np.array_equal(t.numpy(), ins[k]), (name, k)
        for k, (lo, hi) in a1.items():
            n = {"strx": dims[2], "stry": dims[1], "strz": dims[0]}[k]
            assert np.array_equal(synth.uniform((n,), lo, hi, cfg, k), ins[k]), (name, k)
