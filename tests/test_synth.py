"""The seeded generators (synth/) hold no method arithmetic; these pin the properties the
tests and bench rely on: determinism and sliced generation (-m "not gpu")."""
import numpy as np

import synth


def test_device_generator_parts_concatenate_to_the_whole():
    # bench.py under torchrun: rank i of P draws part (i, P); the parts in rank order are
    # the single-process stream (so sliced ingest sees the same global COO)
    kw = dict(m=500, n=300, nnz=10_000, seed=5, n_test=100, chunk=1000, device="cpu")
    (u, v, r), (tu, tv, tr) = synth.powerlaw_device(**kw)
    for P in (2, 3, 7, 16):
        parts = [synth.powerlaw_device(**kw, part=(i, P)) for i in range(P)]
        for a, whole in zip(range(3), (u, v, r)):
            cat = np.concatenate([p[0][a].numpy() for p in parts])
            assert np.array_equal(cat, whole.numpy())
        for p in parts:  # the test set is whole on every part
            assert np.array_equal(p[1][0].numpy(), tu.numpy())
    assert int(u.min()) >= 0 and int(u.max()) < 500 and int(v.max()) < 300


def test_host_generator_is_deterministic():
    a = synth.make(synth.scaled(synth.CONFIGS["c2"], 0.001))
    b = synth.make(synth.scaled(synth.CONFIGS["c2"], 0.001))
    for x, y in zip(a[0] + a[1], b[0] + b[1]):
        assert np.array_equal(x, y)
