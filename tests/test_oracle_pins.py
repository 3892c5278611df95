"""Pins for the CPU oracle against what the paper and mathematics fix (-m "not gpu").

Each test pins the oracle to something other than itself: values printed in the
paper (Fig. 1), hand-computed worked examples, closed forms, invariants,
finite differences and brute force.  A plausible mistake in the oracle (a
dropped term, a wrong sign or index, a transposed operand, new-p instead of
old-p) fails at least one of them; the comment on each test says which.
"""
import math

import numpy as np
import pytest

import golden_io

GOLDEN_MIX = 0x9E3779B97F4A7C15
M64 = (1 << 64) - 1


# ----------------------------------------------------------------- hash spec
def test_splitmix64_published_vectors(orc):
    # SplitMix64 (Steele, Lea, Flood 2014) from state 0: the first four outputs
    # of the reference generator.  orc_splitmix(x) = mix(x + golden), so output i
    # is orc_splitmix(i * golden).  Pins every constant and shift of the mixer.
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F, 0xF88BB8A8724C81EC]
    got = [orc.splitmix((i * GOLDEN_MIX) & M64) for i in range(4)]
    assert got == want


def test_hash_composition_and_uniform(orc):
    # H(seed, tag, a, b) = sm(sm(sm(seed ^ tag<<56) ^ a) ^ b)  (R8)
    for seed, tag, a, b in [(1, 1, 0, 0), (7, 3, 12345, 17), (2**63 + 5, 4, 2**31 - 1, 127)]:
        h = orc.splitmix((seed ^ (tag << 56)) & M64)
        h = orc.splitmix(h ^ a)
        h = orc.splitmix(h ^ b)
        assert orc.hash4(seed, tag, a, b) == h
    # U = (h >> 40) * 2^-24: 0 for h < 2^40 and 1 - 2^-24 for h = 2^64 - 1
    assert orc.uniform(0) == 0.0
    assert orc.uniform(M64) == 1.0 - 2.0 ** -24
    assert orc.uniform(1 << 63) == 0.5


def test_perm_bruteforce(orc):
    # seed 0 = identity; otherwise perm[id] = rank of (H(seed,tag,id,0), id), by Python sorted
    assert list(orc.perm(0, 1, 9)) == list(range(9))
    rng = np.random.default_rng(0)
    for _ in range(50):
        cnt = int(rng.integers(1, 40))
        seed = int(rng.integers(1, 2**63))
        tag = int(rng.integers(1, 3))
        keys = [(orc.hash4(seed, tag, i, 0), i) for i in range(cnt)]
        order = sorted(range(cnt), key=lambda i: keys[i])
        want = np.empty(cnt, np.int32)
        want[order] = np.arange(cnt)
        assert np.array_equal(orc.perm(seed, tag, cnt), want)


# ------------------------------------------------------------ Fig. 1 (paper)
def test_fig1_prediction_matches_printed_Rp(orc):
    # Fig. 1 (L283-L403): R_p = P x Q printed to 2 decimals, all 20 cells.  The
    # oracle's inner product is read through sgd_update with gamma = 0, r = 0
    # (returns e = -p.q).  Pins the dot product and the P (m x k) / Q (n x k)
    # orientation (a transposed Q fails).
    _, P, Q, Rp = golden_io.fig1()
    for i in range(5):
        for j in range(4):
            p, q = P[i].copy(), Q[j].copy()
            pred = -orc.sgd_update(0.0, 0.0, p, q, 0.0)
            assert round(pred + 1e-12, 2) == pytest.approx(Rp[i, j], abs=1e-9), (i, j)


def test_fig1_training_rmse(orc):
    # RMSE over the 12 observed ratings of Fig. 1 with the printed P, Q, computed
    # independently with numpy: SSE = 0.50034114, RMSE = 0.2041938.
    (u, v, r), P, Q, _ = golden_io.fig1()
    pr = np.arange(5, dtype=np.int32)
    pc = np.arange(4, dtype=np.int32)
    sse = float(np.sum((r.astype(np.float64) - np.sum(P[u] * Q[v], axis=1)) ** 2))
    assert sse == pytest.approx(0.50034114, abs=1e-8)
    assert orc.rmse(u, v, r, pr, pc, P, Q) == pytest.approx(math.sqrt(sse / 12), rel=1e-14)
    assert orc.rmse(u, v, r, pr, pc, P, Q) == pytest.approx(0.2041938, abs=1e-7)


def test_single_update_hand_computed(orc):
    # Rating (0, 0, 5.0) of Fig. 1, p = (2.37, 0), q = (2.09, 0.69), lambda = 0.01.
    # By hand: e = 5 - 2.37*2.09 = 0.0467.
    #  gamma = 0.005: p0' = 2.37 + 0.005*(0.0467*2.09 - 0.01*2.37) = 2.370369515
    #                 p1' = 0 + 0.005*(0.0467*0.69) = 0.000161115
    #                 q0' = 2.09 + 0.005*(0.0467*2.37 - 0.01*2.09) = 2.090448895
    #                 q1' = 0.69 + 0.005*(0 - 0.01*0.69) = 0.6899655
    p, q = np.array([2.37, 0.0]), np.array([2.09, 0.69])
    e = orc.sgd_update(0.005, 0.01, p, q, 5.0)
    assert e == pytest.approx(0.0467, abs=1e-12)
    assert p == pytest.approx([2.370369515, 0.000161115], abs=1e-12)
    assert q == pytest.approx([2.090448895, 0.6899655], abs=1e-12)
    # gamma = 0.1 separates the old-p reading (R1) from new-p:
    #   q0' old-p = 2.09 + 0.1*(0.0467*2.37 - 0.0209)  = 2.0989779
    #   q0' new-p = 2.09 + 0.1*(0.0467*2.3773903 - 0.0209) = 2.09901243...
    p, q = np.array([2.37, 0.0]), np.array([2.09, 0.69])
    orc.sgd_update(0.1, 0.01, p, q, 5.0)
    assert p == pytest.approx([2.3773903, 0.0032223], abs=1e-12)
    assert q == pytest.approx([2.0989779, 0.68931], abs=1e-12)
    assert abs(q[0] - 2.0990124) > 3e-5


def test_update_is_minus_gamma_finite_difference_gradient(orc):
    # DESIGN.md R2: step = -gamma * grad f, f = 1/2[(r - p.q)^2 + lambda(|p|^2 + |q|^2)],
    # gradient by central differences in numpy (independent of the oracle).
    rng = np.random.default_rng(3)
    for k in (1, 3, 8):
        p0, q0 = rng.normal(size=k), rng.normal(size=k)
        r, lam, gamma, h = 1.7, 0.3, 0.01, 1e-6

        def f(p, q):
            return 0.5 * ((r - p @ q) ** 2 + lam * (p @ p + q @ q))

        gp = np.array([(f(p0 + h * np.eye(k)[j], q0) - f(p0 - h * np.eye(k)[j], q0)) / (2 * h) for j in range(k)])
        gq = np.array([(f(p0, q0 + h * np.eye(k)[j]) - f(p0, q0 - h * np.eye(k)[j])) / (2 * h) for j in range(k)])
        p, q = p0.copy(), q0.copy()
        orc.sgd_update(gamma, lam, p, q, r)
        np.testing.assert_allclose((p - p0) / -gamma, gp, rtol=1e-6, atol=1e-8)
        np.testing.assert_allclose((q - q0) / -gamma, gq, rtol=1e-6, atol=1e-8)


def test_fig1_end_to_end_epoch(orc):
    # tests/golden/fig1_epoch.txt: partition, sort order, strata order and values.
    g = golden_io.load("fig1_epoch.txt")
    (u, v, r), P0, Q0, _ = golden_io.fig1()
    pr = orc.perm(0, 1, 5)
    S = orc.row_prefix(5, u, pr)
    assert list(S) == [0, 3, 5, 8, 11, 12]
    assert list(orc.bounds(5, 12, S, 2, [0.5, 0.5])) == [int(x) for x in g["bounds_G2"][0]]
    for G, sec in ((1, "sorted_G1_B2"), (2, "sorted_G2_B2")):
        prob = orc.Problem(5, 4, 2, 0.005, 0.01, u, v, r, G=G, Br=2, Bc=2, seed=0)
        want = np.array(g[sec], dtype=np.int64)
        assert np.array_equal(prob.ru, want[:, 3]) and np.array_equal(prob.rv, want[:, 4])
        blk = ((want[:, 0] * 2 + want[:, 1]) * 2 + want[:, 2])
        counts = np.bincount(blk, minlength=G * 4)
        assert np.array_equal(np.diff(prob.off), counts)
    prob = orc.Problem(5, 4, 2, 0.005, 0.01, u, v, r, G=1, Br=2, Bc=2, seed=0)
    prob.set_factors(P0, Q0)
    rm0 = prob.rmse(u, v, r)
    prob.epoch("det", "none")
    P1, Q1 = prob.factors()
    np.testing.assert_allclose(P1, golden_io.matrix(g["P_after"]), atol=1e-10)
    np.testing.assert_allclose(Q1, golden_io.matrix(g["Q_after"]), atol=1e-10)
    assert [rm0, prob.rmse(u, v, r)] == pytest.approx(g["rmse"][0], abs=1e-10)


# --------------------------------------------------- objective / convergence
def _dense_objective(u, v, r, lam, P, Q, m, n):
    # brute force: masked dense residual with a multiplicity mask (duplicates count)
    M = np.zeros((m, n))
    R = np.zeros((m, n))
    np.add.at(M, (u, v), 1.0)
    np.add.at(R, (u, v), r.astype(np.float64))
    pred = P @ Q.T
    # sum over Omega of (r - pq)^2 = sum_cells sum_dups (r_i - pred)^2
    sq = np.zeros((m, n))
    np.add.at(sq, (u, v), (r.astype(np.float64) - pred[u, v]) ** 2)
    reg = lam * (M.sum(axis=1) @ (P * P).sum(axis=1) + M.sum(axis=0) @ (Q * Q).sum(axis=1))
    return sq.sum() + reg


def test_objective_matches_dense_bruteforce(orc):
    import synth
    m, n, k = 7, 6, 3
    u, v, r = synth.tiny(m, n, 30, seed=5)
    rng = np.random.default_rng(1)
    P, Q = rng.normal(size=(m, k)), rng.normal(size=(n, k))
    pr, pc = np.arange(m, dtype=np.int32), np.arange(n, dtype=np.int32)
    got = orc.objective(u, v, r, 0.05, pr, pc, P, Q)
    assert got == pytest.approx(_dense_objective(u, v, r, 0.05, P, Q, m, n), rel=1e-12)


def test_monotone_loss_small_gamma(orc):
    import synth
    m, n, k = 20, 15, 4
    u, v, r = synth.tiny(m, n, 120, seed=11, dup=False)
    prob = orc.Problem(m, n, k, 1e-3, 0.01, u, v, r, G=1, Br=2, Bc=2, seed=9)
    prob.init(4)
    prev = None
    for _ in range(30):
        P, Q = prob.factors()
        L = orc.objective(u, v, r, 0.01, np.arange(m, dtype=np.int32), np.arange(n, dtype=np.int32), P, Q)
        if prev is not None:
            assert L < prev
        prev = L
        prob.epoch("det", "none")


def test_planted_recovery(orc):
    # noise-free rank-4 60 x 40 at 50% density, lambda = 0: train RMSE -> 0
    rng = np.random.default_rng(2)
    m, n, k = 60, 40, 4
    Ps, Qs = rng.uniform(0, 1, (m, k)), rng.uniform(0, 1, (n, k))
    cells = rng.choice(m * n, size=m * n // 2, replace=False)
    u, v = (cells // n).astype(np.int32), (cells % n).astype(np.int32)
    r = np.sum(Ps[u] * Qs[v], axis=1).astype(np.float32)
    prob = orc.Problem(m, n, k, 0.05, 0.0, u, v, r, G=1, Br=1, Bc=1, seed=3)
    prob.init(1)
    first = prob.rmse(u, v, r)
    for _ in range(200):
        prob.epoch("det", "none")
    assert first > 0.3
    assert prob.rmse(u, v, r) < 2e-3


def _gd_step(u, v, r, lam, P, Q, gp, gq):
    # one full-batch gradient step on L/2 (R2, R4): frequency-weighted reg
    E = r.astype(np.float64) - np.sum(P[u] * Q[v], axis=1)
    dP = np.zeros_like(P)
    dQ = np.zeros_like(Q)
    np.add.at(dP, u, E[:, None] * Q[v] - lam * P[u])
    np.add.at(dQ, v, E[:, None] * P[u] - lam * Q[v])
    return P + gp * dP, Q + gq * dQ


@pytest.mark.parametrize("sched,sync,G,Br,Bc", [
    ("det", "none", 1, 3, 3), ("serial", "none", 1, 2, 5), ("det", "ring", 2, 2, 4),
    ("serial", "ring", 3, 1, 3), ("det", "allreduce", 2, 2, 2), ("serial", "allreduce", 3, 1, 1),
])
def test_full_batch_limit(orc, sched, sync, G, Br, Bc):
    # Any serialisation that visits every rating exactly once differs from one
    # full-batch GD step by O(gamma^2): halving gamma quarters the gap.  For the
    # all-reduce mode the Q step is the mean of G replicas, so its first-order
    # term is the GD Q-step divided by G (L549-L557 sync = average).  A dropped
    # or doubled block, a wrong-sign term, or a wrong average fails this.
    import synth
    m, n, k = 9, 7, 3
    u, v, r = synth.tiny(m, n, 40, seed=21)
    rng = np.random.default_rng(4)
    P0, Q0 = rng.uniform(0, 1, (m, k)), rng.uniform(0, 1, (n, k))
    gaps = []
    for gamma in (1e-2, 5e-3, 2.5e-3):
        prob = orc.Problem(m, n, k, gamma, 0.1, u, v, r, G=G, Br=Br, Bc=Bc, seed=13)
        prob.set_factors(P0, Q0)
        prob.epoch(sched, sync)
        P1, Q1 = prob.factors()
        gq = gamma / G if sync == "allreduce" else gamma
        Pg, Qg = _gd_step(u, v, r, 0.1, P0, Q0, gamma, gq)
        first = max(np.abs(P1 - P0).max(), np.abs(Q1 - Q0).max())
        gap = max(np.abs(P1 - Pg).max(), np.abs(Q1 - Qg).max())
        assert gap < 0.2 * first
        gaps.append(gap)
    assert 0.2 < gaps[1] / gaps[0] < 0.3 and 0.2 < gaps[2] / gaps[1] < 0.3


def test_allreduce_g1_equals_none_and_ring_g1_equals_none(orc):
    import synth
    m, n, k = 8, 6, 4
    u, v, r = synth.tiny(m, n, 30, seed=8)
    outs = []
    for sync in ("none", "ring", "allreduce"):
        prob = orc.Problem(m, n, k, 0.05, 0.02, u, v, r, G=1, Br=3, Bc=3, seed=2)
        prob.init(6)
        prob.epoch("det", sync)
        outs.append(prob.factors())
    for P, Q in outs[1:]:
        assert np.array_equal(P, outs[0][0]) and np.array_equal(Q, outs[0][1])


def test_init_range_and_scale(orc):
    m, n, k = 300, 200, 16
    P, Q = orc.init(5, m, n, k, np.arange(m, dtype=np.int32), np.arange(n, dtype=np.int32))
    for X in (P, Q):
        assert X.min() >= 0.0 and X.max() < math.sqrt(1.0 / k)
        assert X.mean() == pytest.approx(0.5 * math.sqrt(1.0 / k), rel=0.02)
        # 24-bit grid: every value is an integer multiple of 2^-24 * sqrt(1/k)
        q = X / (math.sqrt(1.0 / k) * 2.0 ** -24)
        assert np.allclose(q, np.rint(q), atol=1e-6)
    # permuted storage: perm_row maps original id -> stored row
    pr = orc.perm(3, 1, m)
    P2, _ = orc.init(5, m, n, k, pr, np.arange(n, dtype=np.int32))
    assert np.array_equal(P2[pr], P)


def test_init_elements_hand_computed(orc):
    # R5 element by element, from the published SplitMix64 (pinned above) written out here in
    # pure Python: P[u][j] = U(H(seed, 3, u, j)) sqrt(1/k), Q[v][j] = U(H(seed, 4, v, j)) sqrt(1/k).
    # Hand-computed words for seed 7 (u/v = 2, j = 5 and the swapped (5, 2)):
    #   H(7,3,2,5) = 0x0cd83494f4c604e6 -> top 24 bits 841780    -> P[2][5] = 841780 2^-24 sqrt(1/8)
    #   H(7,3,5,2) = 0x566fe5d8ffab1f03 -> 5664741               -> P[5][2]
    #   H(7,4,2,5) = 0xd9d05e5045769262 -> 14274654              -> Q[2][5]
    #   H(7,4,5,2) = 0x43141ffb2255f682 -> 4396063               -> Q[5][2]
    # so swapped (row, column) arguments or swapped tags 3 / 4 change every one of them.
    M, G = (1 << 64) - 1, 0x9E3779B97F4A7C15

    def sm(x):
        z = (x + G) & M
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
        return z ^ (z >> 31)

    assert [sm((i * G) & M) for i in range(1, 3)] == [0x6E789E6AA1B965F4, 0x06C45D188009454F]
    H = lambda seed, tag, a, b: sm(sm(sm(seed ^ (tag << 56)) ^ a) ^ b)  # noqa: E731
    assert H(7, 3, 2, 5) == 0x0CD83494F4C604E6 and H(7, 3, 5, 2) == 0x566FE5D8FFAB1F03
    assert H(7, 4, 2, 5) == 0xD9D05E5045769262 and H(7, 4, 5, 2) == 0x43141FFB2255F682
    k, sc = 8, math.sqrt(1.0 / 8)
    m, n = 9, 7
    pr, pc = orc.perm(11, 1, m), orc.perm(11, 2, n)  # stored permuted: row pr[u] holds user u
    P, Q = orc.init(7, m, n, k, pr, pc)
    assert P[pr[2], 5] == 841780 * 2.0 ** -24 * sc
    assert P[pr[5], 2] == 5664741 * 2.0 ** -24 * sc
    assert Q[pc[2], 5] == 14274654 * 2.0 ** -24 * sc
    assert Q[pc[5], 2] == 4396063 * 2.0 ** -24 * sc
    for u in range(m):
        for j in range(k):
            assert P[pr[u], j] == (H(7, 3, u, j) >> 40) * 2.0 ** -24 * sc
    for v in range(n):
        for j in range(k):
            assert Q[pc[v], j] == (H(7, 4, v, j) >> 40) * 2.0 ** -24 * sc


def test_phased_allreduce_pins(orc):
    # R22: phases = 1 is the plain all-reduce epoch (bit-exact); any phase count keeps
    # the all-reduce first-order limit (P step gamma, Q step gamma / G)
    import synth
    m, n, k, G = 12, 9, 3, 3
    u, v, r = synth.tiny(m, n, 60, seed=31)
    a = orc.Problem(m, n, k, 0.01, 0.1, u, v, r, G=G, Br=4, Bc=2, seed=3)
    b = orc.Problem(m, n, k, 0.01, 0.1, u, v, r, G=G, Br=4, Bc=2, seed=3)
    a.init(2)
    b.init(2)
    a.epoch("serial", "allreduce")
    b.epoch_phased(1)
    assert np.array_equal(a.P, b.P) and np.array_equal(a.Q, b.Q)
    with pytest.raises(ValueError):
        b.epoch_phased(3)  # 4 row blocks cannot be split in 3 rounds
    rng = np.random.default_rng(8)
    P0, Q0 = rng.uniform(0, 1, (m, k)), rng.uniform(0, 1, (n, k))
    gaps = []
    for gamma in (1e-2, 5e-3, 2.5e-3):
        p = orc.Problem(m, n, k, gamma, 0.1, u, v, r, G=G, Br=4, Bc=2, seed=3)
        p.set_factors(P0, Q0)
        p.epoch_phased(4)
        P1, Q1 = p.factors()
        Pg, Qg = _gd_step(u, v, r, 0.1, P0, Q0, gamma, gamma / G)
        gaps.append(max(np.abs(P1 - Pg).max(), np.abs(Q1 - Qg).max()))
    assert 0.2 < gaps[1] / gaps[0] < 0.3 and 0.2 < gaps[2] / gaps[1] < 0.3


def test_round_half_matches_ieee_binary16(orc):
    # Strategy 2 (L1234-L1249): the oracle's binary16 rounding against numpy's
    # IEEE-754 half conversion (round to nearest even) on hand-picked and random values
    cases = [0.0, -0.0, 1.0, 1 / 3, 0.1, 65504.0, 65519.0, 65520.0, 70000.0, 2.0 ** -24, 2.0 ** -25,
             3 * 2.0 ** -26, 2.0 ** -14, 1 + 2.0 ** -11, 1 + 3 * 2.0 ** -11, -2.5e-5, 6.1e-5, 1e-8]
    rng = np.random.default_rng(0)
    cases += list(rng.normal(0, 1, 2000)) + list(rng.uniform(-1e-4, 1e-4, 500)) + list(rng.uniform(-7e4, 7e4, 500))
    for x in cases:
        with np.errstate(over="ignore"):
            want = float(np.float16(x))
        got = orc.round_half(x)
        assert (got == want) or (np.isinf(got) and np.isinf(want) and np.sign(got) == np.sign(want)), (x, got, want)


def test_wire16_epoch_pins(orc):
    # with every Q value already a binary16 number and gamma -> 0 the wire is lossless:
    # the wire16 epoch equals the fp64 epoch; with real updates it differs by at most
    # one binary16 rounding per transfer (relative 2^-11 per stage)
    import synth
    m, n, k, G = 12, 10, 4, 2
    u, v, r = synth.tiny(m, n, 70, seed=41)
    rng = np.random.default_rng(3)
    P0 = rng.uniform(0, 1, (m, k))
    Q0 = np.array([[float(np.float16(x)) for x in row] for row in rng.uniform(0, 1, (n, k))])
    for sync, Br, Bc in (("ring", 2, 4), ("allreduce", 2, 2)):
        a = orc.Problem(m, n, k, 0.0, 0.0, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
        b = orc.Problem(m, n, k, 0.0, 0.0, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
        a.set_factors(P0, Q0)
        b.set_factors(P0, Q0)
        a.epoch("det", sync)
        b.epoch_wire16("det", sync)
        assert np.array_equal(a.Q, b.Q) and np.array_equal(a.P, b.P)
        a = orc.Problem(m, n, k, 0.05, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
        b = orc.Problem(m, n, k, 0.05, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
        a.set_factors(P0, Q0)
        b.set_factors(P0, Q0)
        a.epoch("det", sync)
        b.epoch_wire16("det", sync)
        assert not np.array_equal(a.Q, b.Q)
        assert np.abs(a.Q - b.Q).max() <= 4 * 2.0 ** -11 * np.abs(a.Q).max()
        # every transmitted value is a binary16 number
        assert all(float(np.float16(x)) == x for x in b.Q.ravel())


def test_q16_storage_single_update_hand_computed(orc):
    # Binary16 storage of Q (R26): Q is rounded first, every q write is
    # rounded, P never.  Fig. 1 rating (0, 0, 5.0), p = (2.37, 0), q = (2.09, 0.69),
    # lambda = 0.01.  By hand: rn16(2.09) = 1070 * 2^-9 = 2.08984375,
    # rn16(0.69) = 1413 * 2^-11 = 0.68994140625;  e = 5 - 2.37 * 2.08984375 = 0.0470703125.
    #  gamma = 0.005: q0 = 2.08984375 + 0.005*(0.0470703125*2.37 - 0.0208984375)
    #                    = 2.090297041015625 -> 1070.23 ulps -> 2.08984375 (the step is lost)
    #                 q1 = 0.68994140625 - 0.005*0.0068994140625 = 0.68990690917...
    #                    -> 1412.93 ulps -> 0.68994140625 (lost too: SURVEY H6)
    #                 p0 = 2.37 + 0.005*(0.0470703125*2.08984375 - 0.0237) = 2.370373347991943...
    #                 p1 = 0.005*0.0470703125*0.68994140625 = 0.000162378787994384765625
    #  gamma = 0.1:   q0 = 2.08984375 + 0.0090658203125 = 2.0989095703125 -> 1074.64 -> 2.099609375
    #                 q1 = 0.68994140625 - 0.00068994140625 = 0.68925146484375 -> 1411.59 -> 0.689453125
    u, v, r = np.array([0], np.int32), np.array([0], np.int32), np.array([5.0], np.float32)
    for gamma, want_p, want_q in ((0.005, [2.370373347991943, 0.000162378787994384765625],
                                   [2.08984375, 0.68994140625]),
                                  (0.1, [2.37 + 0.1 * 0.074669598388671875, 0.1 * 0.032475757598876953125],
                                   [2.099609375, 0.689453125])):
        prob = orc.Problem(1, 1, 2, gamma, 0.01, u, v, r, seed=0)
        prob.set_factors(np.array([[2.37, 0.0]]), np.array([[2.09, 0.69]]))
        prob.epoch_q16("serial", "none")
        P, Q = prob.factors()
        assert list(Q[0]) == want_q  # exact: binary16 values
        assert P[0] == pytest.approx(want_p, abs=1e-15)
    # add16 (binary16 add of the rounded increment): gamma = 0.1, increments by hand
    # 0.0090658203125 -> rn16 = 1188.3 * 2^-17 -> 1188 * 2^-17 = 0.0090637207..., and
    # -0.00068994140625 -> -1446.9 * 2^-21 -> -1447 * 2^-21 = -0.000689983367919921875;
    # q0 = rn16(2.08984375 + 0.009063720703125) = rn16(2.098907470703125) = 1074.64 -> 2.099609375
    # q1 = rn16(0.68994140625 - 0.000689983367919921875) = 1411.59 ulps -> 0.689453125
    # (same stored values here: the rounded increment moves each sum by < 0.01 ulp)
    prob = orc.Problem(1, 1, 2, 0.1, 0.01, u, v, r, seed=0)
    prob.set_factors(np.array([[2.37, 0.0]]), np.array([[2.09, 0.69]]))
    prob.epoch_q16("serial", "none", add16=True)
    assert list(prob.factors()[1][0]) == [2.099609375, 0.689453125]
    assert float(np.float16(0.0090658203125)) == 1188 * 2.0 ** -17
    assert float(np.float16(-0.00068994140625)) == -1447 * 2.0 ** -21


def test_q16_storage_epoch_invariants(orc):
    # every stored q is a binary16 number, P is not rounded, and the binary16 epoch stays
    # within a few binary16 ulps of the fp64 epoch on a small problem
    import synth
    m, n, k = 30, 20, 8
    u, v, r = synth.tiny(m, n, 300, seed=7)
    rng = np.random.default_rng(5)
    P0, Q0 = rng.uniform(0, 1, (m, k)), rng.uniform(0, 1, (n, k))
    for sched, sync, G, Br, Bc in (("det", "none", 1, 3, 3), ("serial", "none", 1, 1, 1),
                                    ("det", "ring", 2, 2, 4), ("det", "allreduce", 2, 3, 3)):
        a = orc.Problem(m, n, k, 0.01, 0.05, u, v, r, G=G, Br=Br, Bc=Bc, seed=9)
        b = orc.Problem(m, n, k, 0.01, 0.05, u, v, r, G=G, Br=Br, Bc=Bc, seed=9)
        a.set_factors(P0, Q0)
        b.set_factors(P0, Q0)
        a.epoch(sched, sync)
        b.epoch_q16(sched, sync)
        if sync != "allreduce":  # the mean of binary16 copies is not itself rounded
            assert all(float(np.float16(x)) == x for x in b.Q.ravel())
        assert not all(float(np.float16(x)) == x for x in b.P.ravel())
        assert 0 < np.abs(a.Q - b.Q).max() <= 8 * 2.0 ** -11 * np.abs(a.Q).max()
        assert np.abs(a.P - b.P).max() <= 8 * 2.0 ** -11 * np.abs(a.P).max()
        c = orc.Problem(m, n, k, 0.01, 0.05, u, v, r, G=G, Br=Br, Bc=Bc, seed=9)
        c.set_factors(P0, Q0)
        c.epoch_q16(sched, sync, add16=True)
        assert 0 < np.abs(b.Q - c.Q).max() <= 8 * 2.0 ** -11 * np.abs(b.Q).max()


def _f16_down(x):
    """largest binary16 value <= |x| (numpy's IEEE conversion, stepped toward zero)"""
    a = abs(float(x))
    d = np.float16(a)
    if float(d) > a:
        d = np.nextafter(d, np.float16(0))
    return float(d)


def test_sr_rounding_definition(orc):
    # R27: one of the two binary16 neighbours; on-grid values are kept for every R;
    # R = 0 truncates toward zero; averaging over all 2^13 random inputs reproduces any
    # fp32 value of the normal binary16 range exactly (13 dropped bits), i.e. unbiased
    rng = np.random.default_rng(11)
    xs = np.concatenate([rng.uniform(-3, 3, 40), rng.uniform(2.0 ** -14, 1e-3, 20),
                         rng.uniform(100, 60000, 20)]).astype(np.float32)
    R = np.arange(8192)
    for x in xs:
        x = float(x)
        dn = _f16_down(x)
        up = float(np.nextafter(np.float16(dn), np.float16(np.inf)))
        ys = np.array([orc.round_half_sr(x, int(r)) for r in R[::64]] + [orc.round_half_sr(x, 8191)])
        assert set(np.abs(ys)) <= {dn, up}, x
        assert abs(orc.round_half_sr(x, 0)) == dn
        full = np.array([orc.round_half_sr(x, int(r)) for r in R])
        assert full.mean() == x  # exact: the fraction past dn is a multiple of 2^-13 ulp
    for h in (np.float16(0.3), np.float16(-2.5), np.float16(6e-5), np.float16(1e-7)):
        for r in (0, 1, 4095, 8191):
            assert orc.round_half_sr(float(h), r) == float(h)


def test_sr_word_is_the_stated_hash(orc):
    # lowbias32 inverted step by step (modular inverses of the odd multipliers, xorshift
    # inverses) must give back i*0x9E3779B1 + t*0x85EBCA77 + c*0xC2B2AE3D mod 2^32 for even c;
    # an odd pair's word is its even neighbour's times 0x9E3779B1 (R27): undo that first
    M = 2 ** 32
    inv1, inv2, inv_phi = pow(0x846CA68B, -1, M), pow(0x7FEB352D, -1, M), pow(0x9E3779B1, -1, M)
    rng = np.random.default_rng(2)
    for _ in range(300):
        i, t, c = int(rng.integers(0, 2 ** 40)), int(rng.integers(0, 2 ** 32)), int(rng.integers(0, 2 ** 12))
        x = orc.sr_word(i, t, c)
        if c % 2:
            x = (x * inv_phi) % M
            c -= 1
        x ^= x >> 16
        x = (x * inv1) % M
        x ^= (x >> 15) ^ (x >> 30)
        x = (x * inv2) % M
        x ^= x >> 16
        assert x == (i * 0x9E3779B1 + t * 0x85EBCA77 + c * 0xC2B2AE3D) % M
    # the two 13-bit fields are uniform
    w = np.array([orc.sr_word(i, 3, c) for i in range(2000) for c in range(8)], dtype=np.uint64)
    for f in (w & 0x1FFF, (w >> 16) & 0x1FFF):
        h = np.bincount((f >> 9).astype(np.int64), minlength=16)  # 16 bins of 512
        exp = len(f) / 16
        assert ((h - exp) ** 2 / exp).sum() < 50  # chi-square, 15 dof (p ~ 1e-5)


def test_sr_epoch_single_update_and_invariants(orc):
    # Fig. 1 rating (0, 0, 5.0), gamma = 0.005 (see test_q16_storage_single_update_hand_computed):
    # q0 + dq0 = 2.090297041015625 lies 0.232085 ulps (2^-9) above 2.08984375, so it
    # rounds up iff R13 >= 8192 * (1 - 0.232085) = 6290.8; q1 + dq1 = 0.6899069091796875
    # lies 0.929350 ulps (2^-11) above 0.689453125, up iff R13 >= 8192 * 0.070650 = 578.8
    u, v, r = np.array([0], np.int32), np.array([0], np.int32), np.array([5.0], np.float32)
    for t in range(6):
        w = orc.sr_word(0, t, 0)
        prob = orc.Problem(1, 1, 2, 0.005, 0.01, u, v, r, seed=0)
        prob.set_factors(np.array([[2.37, 0.0]]), np.array([[2.09, 0.69]]))
        prob.epoch_q16("serial", "none", sr=True, t=t)
        q = prob.factors()[1][0]
        assert q[0] == (2.08984375 + 2.0 ** -9 if (w & 0x1FFF) >= 6291 else 2.08984375)
        assert q[1] == (0.689453125 + 2.0 ** -11 if ((w >> 16) & 0x1FFF) >= 579 else 0.689453125)
    # every stored q is binary16; the SR epoch tracks the fp64 epoch within a few ulps; a
    # different epoch counter gives different roundings
    import synth
    m, n, k = 30, 20, 8
    u, v, r = synth.tiny(m, n, 300, seed=7)
    rng = np.random.default_rng(5)
    P0, Q0 = rng.uniform(0, 1, (m, k)), rng.uniform(0, 1, (n, k))
    res = []
    for t in (0, 1):
        a = orc.Problem(m, n, k, 0.01, 0.05, u, v, r, G=1, Br=3, Bc=3, seed=9)
        b = orc.Problem(m, n, k, 0.01, 0.05, u, v, r, G=1, Br=3, Bc=3, seed=9)
        a.set_factors(P0, Q0)
        b.set_factors(P0, Q0)
        a.epoch("det", "none")
        b.epoch_q16("det", "none", sr=True, t=t)
        assert all(float(np.float16(x)) == x for x in b.Q.ravel())
        assert 0 < np.abs(a.Q - b.Q).max() <= 8 * 2.0 ** -11 * np.abs(a.Q).max()
        res.append(b.Q.copy())
    assert not np.array_equal(res[0], res[1])
