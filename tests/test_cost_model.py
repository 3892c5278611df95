"""Section 3.2 time cost model (Eq. 1-5) and the DP1/DP2 choice (-m "not gpu").

The oracle is pinned by hand arithmetic; the library's host planner (no device
needed) must agree with the oracle."""
import numpy as np
import pytest


def test_oracle_cost_model_hand_computed(orc):
    # p = 2, B = (2, 1) GB/s, nnz = 1000, k = 4 -> 16k+4 = 68 B/rating
    # T_e = (3.4e-5, 6.8e-5) s; Eq. 6: x = (2/3, 1/3); both computing terms 2.2667e-5 s
    # Strategy 1: D = n = 20; Eq. 2 comm = 2 * 4 B * 4 * 20 / 1e9 = 6.4e-7 s
    # Eq. 3: T_sync = 3 * 1 * 4 * 4 * 20 / 1e9 = 9.6e-7 s; ratio 24.3 >= 10 -> DP1, T = max T_i
    x, Ti, Ts, T, br = orc.cost_model(10, 20, 1000, 4, [2e9, 1e9], [1e9, 1e9], 1e9)
    np.testing.assert_allclose(x, [2 / 3, 1 / 3], rtol=1e-14)
    np.testing.assert_allclose(Ti, [68000 / 3e9 + 6.4e-7] * 2, rtol=1e-12)
    assert Ts == pytest.approx(9.6e-7, rel=1e-14)
    assert br == 1 and T == pytest.approx(Ti.max(), rel=1e-15)
    # a server 10x slower: ratio 2.4 < 10 -> DP2, T = max T_i + T_sync (Eq. 5)
    x, Ti, Ts, T, br = orc.cost_model(10, 20, 1000, 4, [2e9, 1e9], [1e9, 1e9], 1e8)
    assert br == 2 and T == pytest.approx(Ti.max() + 9.6e-6, rel=1e-12)
    # without Strategy 1 the moved parameters are m + n = 30 (Eq. 2 as printed)
    _, Ti2, Ts2, _, _ = orc.cost_model(10, 20, 1000, 4, [2e9, 1e9], [1e9, 1e9], 1e9, q_only=0)
    assert Ts2 == pytest.approx(1.44e-6, rel=1e-14)
    assert Ti2[0] - Ti[0] == pytest.approx(2 * 4 * 4 * 10 / 1e9, rel=1e-9)


def test_library_cost_model_matches_oracle(orc):
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_huangylhbl21_b200 as hc
    rng = np.random.default_rng(5)
    for _ in range(50):
        p = int(rng.integers(1, 9))
        B = rng.uniform(30e9, 7000e9, p)
        Bbus = rng.uniform(10e9, 900e9, p)
        Bs = float(rng.uniform(50e9, 7000e9))
        m, n = int(rng.integers(1, 10**8)), int(rng.integers(1, 10**6))
        nnz, k = int(rng.integers(1, 4 * 10**9)), int(rng.choice([16, 32, 128]))
        t, q, e = int(rng.integers(1, 4)), int(rng.integers(0, 2)), int(rng.choice([2, 4]))
        lam = float(rng.uniform(1, 20))
        xo, To, Tso, TTo, bro = orc.cost_model(m, n, nnz, k, B, Bbus, Bs, t, q, e, lam)
        xl, Tl, Tsl, TTl, brl = hc.cost_model(m, n, nnz, k, B, Bbus, Bs, t, bool(q), e, lam)
        np.testing.assert_allclose(xl, xo, rtol=1e-15)
        np.testing.assert_allclose(Tl, To, rtol=1e-15)
        assert Tsl == pytest.approx(Tso, rel=1e-15) and TTl == pytest.approx(TTo, rel=1e-15)
        assert brl == {1: "DP1", 2: "DP2"}[bro]
    with pytest.raises(hc.HccmfError):
        hc.cost_model(1, 1, 1, 4, [0.0], [1.0], 1.0)
