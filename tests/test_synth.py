"""Pins for the shared seeded generator (synth/) — golden vectors, not the method."""
import json
import os

import numpy as np

import synth

G = os.path.join(os.path.dirname(__file__), "golden")


def test_splitmix64_golden_vectors():
    gv = json.load(open(os.path.join(G, "splitmix64_vectors.json")))
    assert int(synth.splitmix64(0, np.array([0]))[0]) == int(gv["seed0_first_u64"], 16)
    got = synth.uniform_from_index(gv["seed"], np.array(gv["index"]))
    assert got.tolist() == gv["value"]


def test_grid_is_indexed_by_linear_padded_index():
    g = synth.grid((5, 7), 20240101, chunk=3)
    assert g[0, 0] == 1.3247442238784974 and g[0, 2] == 1.0931883103130873
    assert g.min() >= 0.5 and g.max() < 1.5


def test_rsym_weights_symmetry_and_normalisation():
    for d, h in [(2, 1), (2, 3), (3, 1), (2, 4)]:
        W = synth.rsym_weights(d, h, 3)
        assert abs(W.sum() - 1) < 1e-15 and W.min() > 0
        for ax in range(d):
            assert np.array_equal(W, np.flip(W, ax))
        assert np.array_equal(W, np.swapaxes(W, 0, 1))
    # class count for 2D h=3 is 10
    assert len(np.unique(synth.rsym_weights(2, 3, 3))) == 10
    assert len(np.unique(synth.rsym_weights(3, 1, 3))) == 4


def test_presets_sum_to_one():
    assert synth.preset("heat2d").sum() == 1.0 and synth.preset("heat3d").sum() == 1.0


def test_grid_torch_is_bit_identical():
    import torch
    g = synth.grid_torch((37, 41), 20240101, device="cpu", chunk=100).numpy()
    assert np.array_equal(g, synth.grid((37, 41), 20240101))
