"""Pins for the oracle's partitioner (section 3.3) and blocker (L546, L1472-L1474).

Brute force on tiny inputs with Python's sorted/min (textbook routines), the
DP0 closed form (Eq. 6), Theorem 1's equalisation, and invariants.
"""
import math

import numpy as np
import pytest


def _llround(x):
    return int(math.floor(x + 0.5))  # x >= 0: round half away from zero


def _bruteforce_partition(m, n, u, v, G, Br, Bc, x, perm_row, perm_col, seed=0, orc=None):
    cnt = np.bincount(perm_row[u], minlength=m) if len(u) else np.zeros(m, int)
    S = [0]
    for c in cnt:
        S.append(S[-1] + int(c))
    b = [0]
    cum = 0.0
    for s in range(1, G):
        cum += x[s - 1]
        T = _llround(len(u) * cum)
        b.append(min(range(b[-1], m + 1), key=lambda r_: (abs(S[r_] - T), r_)))
    b.append(m)
    recs = []
    for i in range(len(u)):
        up, vp = int(perm_row[u[i]]), int(perm_col[v[i]])
        s = max(j for j in range(G) if b[j] <= up < b[j + 1])
        rb = (up - b[s]) * Br // (b[s + 1] - b[s])
        cb = vp * Bc // n
        c0, c1 = -(-cb * n // Bc), -(-(cb + 1) * n // Bc)
        rot = orc.hash4(seed, 5, up, 0) % (c1 - c0) if seed else 0
        recs.append((((s * Br + rb) * Bc + cb), up, (vp - c0 + rot) % (c1 - c0), i, vp))
    recs.sort()
    off = [0] * (G * Br * Bc + 1)
    for rec in recs:
        off[rec[0] + 1] += 1
    for j in range(G * Br * Bc):
        off[j + 1] += off[j]
    return S, b, recs, off


def test_partition_and_sort_bruteforce(orc):
    import synth
    rng = np.random.default_rng(1234)
    for trial in range(400):
        m, n = int(rng.integers(1, 9)), int(rng.integers(1, 9))
        nnz = int(rng.integers(0, 65))
        G = int(rng.integers(1, min(m, 4) + 1))
        Br, Bc = int(rng.integers(1, 5)), int(rng.integers(1, 5))
        seed = 0 if trial % 4 == 0 else int(rng.integers(1, 2**62))
        u, v, r = synth.tiny(m, n, nnz, seed=trial)
        x = rng.dirichlet(np.ones(G)) if trial % 2 else np.full(G, 1.0 / G)
        pr, pc = orc.perm(seed, 1, m), orc.perm(seed, 2, n)
        S, b, recs, off = _bruteforce_partition(m, n, u, v, G, Br, Bc, x, pr, pc, seed, orc)
        assert list(orc.row_prefix(m, u, pr)) == S
        ob = orc.bounds(m, nnz, np.array(S, np.int64), G, x)
        assert list(ob) == b
        if any(b[s + 1] == b[s] for s in range(G)) and nnz:
            # an empty shard with ratings elsewhere is fine; the blocker never
            # divides by its zero row count because no record lands in it
            pass
        ou, ov, orr, ooff = orc.block_sort(m, n, u, v, r, G, Br, Bc, ob, pr, pc, seed)
        assert list(ooff) == off
        assert list(ou) == [t[1] for t in recs] and list(ov) == [t[4] for t in recs]
        assert np.array_equal(orr, r[[t[3] for t in recs]])


def test_partition_invariants_medium(orc):
    import synth
    m, n, nnz = 500, 300, 20000
    (u, v, r), _ = synth.powerlaw(m, n, nnz, seed=3, n_test=0)
    for seed in (0, 99):
        pr, pc = orc.perm(seed, 1, m), orc.perm(seed, 2, n)
        assert sorted(pr) == list(range(m)) and sorted(pc) == list(range(n))
        S = orc.row_prefix(m, u, pr)
        cnt = np.diff(S)
        for G in (1, 2, 3, 8):
            x = np.full(G, 1.0 / G)
            b = orc.bounds(m, nnz, S, G, x)
            assert b[0] == 0 and b[-1] == m and np.all(np.diff(b) >= 0)
            cum = np.cumsum(x)
            for s in range(1, G):
                assert abs(S[b[s]] - _llround(nnz * cum[s - 1])) <= cnt.max()
            ou, ov, orr, off = orc.block_sort(m, n, u, v, r, G, 4, 5, b, pr, pc, seed)
            assert off[-1] == nnz
            # multiset preserved
            a = np.sort(np.stack([ou, ov, orr.view(np.int32)]), axis=1)
            want = np.sort(np.stack([pr[u], pc[v], r.view(np.int32)]), axis=1)
            assert np.array_equal(np.sort(ou), np.sort(pr[u]))
            assert np.array_equal(np.sort(orr), np.sort(r))
            # row-sorted within each block (rows contiguous, each row a rotation of the
            # block's columns, R21); every record inside its block's ranges
            for blk in range(G * 20):
                lo, hi = off[blk], off[blk + 1]
                s, rem = divmod(blk, 20)
                rb, cb = divmod(rem, 5)
                assert np.all(np.diff(ou[lo:hi]) >= 0)
                assert np.all((ou[lo:hi] >= b[s]) & (ou[lo:hi] < b[s + 1]))
                assert np.all(ov[lo:hi] * 5 // n == cb)
            del a, want


def test_dp0_eq6_closed_form(orc):
    # Eq. 6: x_i = 1 / sum_j (T_i,e / T_j,e)  ==  (1/T_i) / sum_j (1/T_j); sum = 1;
    # Theorem 1 with equal b: a_i x_i equal for all i (L961-L964)
    t = np.array([1.0, 2.0, 4.0, 0.5])
    x = orc.dp0(t)
    np.testing.assert_allclose(x, (1 / t) / np.sum(1 / t), rtol=1e-15)
    assert x.sum() == pytest.approx(1.0, abs=1e-15)
    np.testing.assert_allclose(t * x, (t * x)[0], rtol=1e-14)
    # homogeneous GPUs -> 1/G
    np.testing.assert_allclose(orc.dp0(np.full(8, 3.3)), np.full(8, 1 / 8), rtol=1e-15)


def test_theorem1_affine_equalisation(orc):
    # Theorem 1 (L924-L954): argmin max(a_i x_i + b_i) s.t. sum x = 1 equalises
    # a_i x_i + b_i; checked against a brute-force grid search for p = 3
    a = np.array([2.0, 3.0, 5.0])
    b = np.array([0.1, 0.3, 0.2])
    x = orc.dp0_affine(a, b)
    assert x.sum() == pytest.approx(1.0, abs=1e-14)
    np.testing.assert_allclose(a * x + b, (a * x + b)[0], rtol=1e-12)
    best = min(((max(a[0] * i / 400 + b[0], a[1] * j / 400 + b[1], a[2] * (400 - i - j) / 400 + b[2]), i, j)
                for i in range(401) for j in range(401 - i)))
    assert max(a * x + b) <= best[0] + 1e-12
    assert max(a * x + b) == pytest.approx(best[0], abs=0.01)
    # a worker whose communication alone exceeds the optimum gets no data
    x = orc.dp0_affine(np.array([1.0, 1.0]), np.array([0.0, 5.0]))
    np.testing.assert_allclose(x, [1.0, 0.0])


def test_dp1_compensation(orc):
    # Algorithm 1 (L1025-L1142), GPU-only generalisation (R11):
    # already balanced within 10% -> unchanged, zero rounds
    x0 = np.array([0.25, 0.25, 0.25, 0.25])
    x, it = orc.dp1(x0, np.array([1.0, 1.05, 0.97, 1.02]))
    assert it == 0 and np.array_equal(x, x0)
    # imbalanced: the linear-bandwidth model (L1013-L1016) balances in one round
    t = np.array([1.0, 2.0, 1.0, 1.0])
    x, it = orc.dp1(x0, t)
    assert it == 1 and x.sum() == pytest.approx(1.0, abs=1e-15)
    pred = t * x / x0  # predicted times at the new partition
    np.testing.assert_allclose(pred, pred[0], rtol=1e-12)
    assert x[1] < x[0]


def test_dp2_hidden_sync_ramp(orc):
    # Eq. 7 (L1166): T_(i+-n),c = T_i,c +- n T_i,sync around the median shard
    x0 = np.full(5, 0.2)
    t = np.full(5, 1.0)
    x = orc.dp2(x0, t, 0.1)
    assert x.sum() == pytest.approx(1.0, abs=1e-15)
    pred = t * x / x0
    d = np.diff(pred)
    np.testing.assert_allclose(d, d[0], rtol=1e-12)
    # ramp step relative to the median time equals t_sync / T_med
    assert d[0] / pred[2] == pytest.approx(0.1, rel=1e-12)


# ----------------------------------------- degree-balanced column blocks (R30)
def _col_blocks(n, B):
    return [(-(-c * n // B), -(-(c + 1) * n // B)) for c in range(B)]


def test_balanced_perm_hand_example(orc):
    # n = 5 items, B = 2 column blocks (slots [0, 3) and [3, 5)); degrees
    # item: 0 1 2 3 4 -> 1 5 3 5 2.  Order (degree desc, id asc): 1 (5), 3 (5), 2 (3), 4 (2), 0 (1).
    #   1 -> block 0 (loads 0, 0: tie -> lowest)     slot 0      loads (5, 0)
    #   3 -> block 1                                  slot 3      loads (5, 5)
    #   2 -> block 0 (tie)                            slot 1      loads (8, 5)
    #   4 -> block 1                                  slot 4      loads (8, 7), block 1 full
    #   0 -> block 0 (only free slot)                 slot 2      loads (9, 7)
    v = np.array([0] + [1] * 5 + [2] * 3 + [3] * 5 + [4] * 2, np.int32)
    assert list(orc.perm_balanced(5, v, 2)) == [2, 0, 1, 3, 4]
    # B = 1: one block, slots in degree order
    assert list(orc.perm_balanced(5, v, 1)) == [4, 0, 2, 1, 3]


def test_balanced_perm_invariants(orc):
    # a permutation whose blocks have exactly their a4 widths and whose loads add up to nnz;
    # on skewed data its heaviest block is lighter than the hash shuffle's in aggregate (a
    # reversed order or a max-load rule would make it heavier)
    rng = np.random.default_rng(3)
    tot_bal = tot_hash = 0
    for trial in range(60):
        n = int(rng.integers(1, 200))
        B = int(rng.integers(1, min(n, 40) + 1))
        nnz = int(rng.integers(0, 3000))
        v = (rng.zipf(1.5, nnz) % n).astype(np.int32) if trial % 2 else rng.integers(0, n, nnz).astype(np.int32)
        pc = orc.perm_balanced(n, v, B)
        assert np.array_equal(np.sort(pc), np.arange(n))
        deg = np.bincount(v, minlength=n)
        widths = [b - a for a, b in _col_blocks(n, B)]
        loads = np.array([deg[(pc >= a) & (pc < b)].sum() for a, b in _col_blocks(n, B)])
        assert loads.sum() == nnz and sum(widths) == n
        ph = orc.perm(7, 2, n)
        tot_bal += loads.max()
        tot_hash += max(deg[(ph >= a) & (ph < b)].sum() for a, b in _col_blocks(n, B))
    assert tot_bal < tot_hash, (tot_bal, tot_hash)


def test_balanced_perm_partition_is_a_valid_block_sort(orc):
    # Problem(col_balance=1): the sort invariants of section 8(c) c1.4 hold with the new
    # column ids (every rating kept once, each record inside its column block)
    u, v, r = synth_tiny()
    for B in (1, 2, 5):
        prob = orc.Problem(40, 30, 4, 0.01, 0.01, u, v, r, G=1, Br=B, Bc=B, seed=3, col_balance=1)
        assert np.array_equal(np.sort(prob.perm_col), np.arange(30))
        cb = (prob.rv.astype(np.int64) * B) // 30
        blocks = np.repeat(np.arange(B * B), np.diff(prob.off))
        assert np.array_equal(blocks % B, cb)
        assert sorted(zip(prob.perm_row[u], prob.perm_col[v])) == sorted(zip(prob.ru, prob.rv))


def synth_tiny():
    import synth
    return synth.tiny(40, 30, 500, seed=11)


def test_rotated_row_order_hand_computed(orc):
    # R21 with a non-zero seed, by hand: one user (m = 1, so u' = 0), items 0..4 rated 1..5.
    # perm_col(seed 11): H(11, 2, v, 0) = aa53.., 0b7b.., 9a38.., abbb.., 8fbc.. (v = 0..4) -> ranks
    # v' = [3, 0, 2, 4, 1]; H(11, 5, 0, 0) = 0x21917a0b7eba4497: mod 5 = 2, mod 3 = 2, mod 2 = 1.
    # One block (w = 5): o = (v' + 2) mod 5 -> the row runs v' = 3, 4, 0, 1, 2 (items 0, 3, 1, 4, 2).
    # Two column blocks: [0, 3) with rotation 2 -> o = (v' + 2) mod 3 -> v' 1, 2, 0; [3, 5) with rotation 1
    # -> o = (v' - 3 + 1) mod 2 -> v' 4, 3.
    u = np.zeros(5, np.int32)
    v = np.arange(5, dtype=np.int32)
    r = np.arange(1, 6, dtype=np.float32)
    p1 = orc.Problem(1, 5, 4, 0.01, 0.01, u, v, r, G=1, Br=1, Bc=1, seed=11)
    assert list(p1.perm_col) == [3, 0, 2, 4, 1]
    assert list(p1.rv) == [3, 4, 0, 1, 2] and list(p1.rr) == [1.0, 4.0, 2.0, 5.0, 3.0]
    p2 = orc.Problem(1, 5, 4, 0.01, 0.01, u, v, r, G=1, Br=1, Bc=2, seed=11)
    assert list(p2.rv) == [1, 2, 0, 4, 3] and list(p2.off) == [0, 3, 5]
    p0 = orc.Problem(1, 5, 4, 0.01, 0.01, u, v, r, G=1, Br=1, Bc=1, seed=0)  # seed 0: plain order
    assert list(p0.rv) == [0, 1, 2, 3, 4]
