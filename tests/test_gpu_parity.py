"""GPU parity: the CUDA path (through the C ABI) vs the oracle, element by element.

Bars: bit-exact for the shuffle, partition and sort;
max-abs <= 1e-4 for factors after one deterministic epoch (north_star); rel 1e-6
for RMSE on identical factors; test RMSE within 0.005 of the oracle's for the
Hogwild and multi-shard modes.
"""
import numpy as np
import pytest

import bands
import golden_io
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_huangylhbl21_b200 as p
    return p


def _gpu_problem(pkg, m, n, k, gamma, lam, u, v, r, G=1, Br=1, Bc=1, seed=0, strategy="DP0", x=None, t_meas=None,
                 t_sync=0.0, col_balance=False):
    mdl = pkg.Model(m, n, k, gamma, lam)
    mdl.load(u, v, r)
    mdl.partition(G, (Br, Bc), strategy, seed=seed, x=x, t_meas=t_meas, t_sync=t_sync, col_balance=col_balance)
    return mdl


def _check_partition(mdl, prob):
    b, off, pr, pc = mdl.get_partition()
    assert np.array_equal(pr, prob.perm_row)
    assert np.array_equal(pc, prob.perm_col)
    assert np.array_equal(b, prob.b)
    assert np.array_equal(off, prob.off)
    gu, gv, gr = mdl.records()
    assert np.array_equal(gu, prob.ru)
    assert np.array_equal(gv, prob.rv)
    assert np.array_equal(gr.view(np.int32), prob.rr.view(np.int32))


# ------------------------------------------------------------------ Fig. 1
def test_fig1_end_to_end(pkg, orc):
    g = golden_io.load("fig1_epoch.txt")
    (u, v, r), P0, Q0, _ = golden_io.fig1()
    # k = 2 is not a multiple of 4: the library rejects it, so the fixture runs at
    # k = 4 with the two extra latent columns zero (they stay exactly zero).
    P4 = np.zeros((5, 4), np.float32)
    Q4 = np.zeros((4, 4), np.float32)
    P4[:, :2], Q4[:, :2] = P0, Q0
    mdl = _gpu_problem(pkg, 5, 4, 4, 0.005, 0.01, u, v, r, G=1, Br=2, Bc=2)
    mdl.set_factors(P4, Q4)
    rm0 = mdl.rmse(u, v, r)
    mdl.train_epoch("det", "none")
    P, Q = mdl.factors()
    assert np.all(P[:, 2:] == 0) and np.all(Q[:, 2:] == 0)
    np.testing.assert_allclose(P[:, :2], golden_io.matrix(g["P_after"]), atol=1e-6)
    np.testing.assert_allclose(Q[:, :2], golden_io.matrix(g["Q_after"]), atol=1e-6)
    assert rm0 == pytest.approx(g["rmse"][0][0], abs=1e-6)
    assert mdl.rmse(u, v, r) == pytest.approx(g["rmse"][0][1], abs=1e-6)
    b, off, _, _ = mdl.get_partition()
    assert list(b) == [0, 5]
    mdl2 = _gpu_problem(pkg, 5, 4, 4, 0.005, 0.01, u, v, r, G=2, Br=2, Bc=2)
    assert list(mdl2.get_partition()[0]) == [int(x) for x in g["bounds_G2"][0]]


# -------------------------------------------------------- partition (a2-a4)
def test_partition_bitexact_tiny_bruteforce(pkg, orc):
    rng = np.random.default_rng(7)
    for trial in range(120):
        m, n = int(rng.integers(1, 12)), int(rng.integers(1, 12))
        nnz = int(rng.integers(0, 80))
        G = int(rng.integers(1, min(m, 4) + 1))
        Br, Bc = int(rng.integers(1, 5)), int(rng.integers(1, 5))
        seed = 0 if trial % 3 == 0 else int(rng.integers(1, 2**62))
        u, v, r = synth.tiny(m, n, nnz, seed=trial)
        x = rng.dirichlet(np.ones(G)) if trial % 2 else None
        prob = orc.Problem(m, n, 4, 0.01, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=seed, x=x)
        mdl = _gpu_problem(pkg, m, n, 4, 0.01, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=seed, x=x)
        _check_partition(mdl, prob)
        mdl.close()


@pytest.mark.parametrize("G,Br,Bc,seed", [(1, 1, 1, 3), (1, 16, 16, 3), (4, 8, 32, 11), (3, 5, 7, 0)])
def test_partition_bitexact_powerlaw(pkg, orc, G, Br, Bc, seed):
    cfg = synth.scaled(synth.CONFIGS["c2"], 0.02)
    (u, v, r), _ = synth.powerlaw(cfg.m, cfg.n, cfg.nnz, seed=cfg.seed, n_test=0, scale="half")
    prob = orc.Problem(cfg.m, cfg.n, 8, 0.005, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=seed)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, 8, 0.005, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=seed)
    _check_partition(mdl, prob)


def test_partition_dp_strategies_bitexact(pkg, orc):
    cfg = synth.scaled(synth.CONFIGS["c2"], 0.01)
    (u, v, r), _ = synth.powerlaw(cfg.m, cfg.n, cfg.nnz, seed=5, n_test=0)
    G = 4
    t = np.array([1.0, 1.6, 0.9, 1.2])
    x0 = np.full(G, 0.25)
    cases = [("DP0", orc.dp0(t), dict(t_meas=t)),
             ("DP1", orc.dp1(x0, t)[0], dict(x=x0, t_meas=t)),
             ("DP2", orc.dp2(x0, t, 0.05), dict(x=x0, t_meas=t, t_sync=0.05))]
    for name, xo, kw in cases:
        mdl = _gpu_problem(pkg, cfg.m, cfg.n, 8, 0.005, 0.01, u, v, r, G=G, Br=2, Bc=8, seed=9, strategy=name, **kw)
        assert np.array_equal(mdl.fractions(), xo), name
        prob = orc.Problem(cfg.m, cfg.n, 8, 0.005, 0.01, u, v, r, G=G, Br=2, Bc=8, seed=9, x=xo)
        _check_partition(mdl, prob)


def test_partition_edge_cases(pkg, orc):
    # nnz = 0, m = 1, n = 1, all ratings in one cell, G = m
    for (m, n, nnz, G, Br, Bc) in [(5, 4, 0, 1, 2, 2), (1, 7, 20, 1, 1, 3), (9, 1, 20, 3, 2, 1), (6, 6, 30, 6, 1, 1)]:
        u, v, r = synth.tiny(m, n, nnz, seed=m * 100 + n)
        prob = orc.Problem(m, n, 4, 0.01, 0.0, u, v, r, G=G, Br=Br, Bc=Bc, seed=2)
        mdl = _gpu_problem(pkg, m, n, 4, 0.01, 0.0, u, v, r, G=G, Br=Br, Bc=Bc, seed=2)
        _check_partition(mdl, prob)
        mdl.init(1)
        mdl.train_epoch("hogwild", "none" if G == 1 else "ring") if Bc % G == 0 else None
    u = np.zeros(50, np.int32)
    v = np.zeros(50, np.int32)
    r = np.linspace(1, 5, 50).astype(np.float32)
    prob = orc.Problem(3, 3, 4, 0.01, 0.0, u, v, r, G=1, Br=2, Bc=2, seed=4)
    _check_partition(_gpu_problem(pkg, 3, 3, 4, 0.01, 0.0, u, v, r, G=1, Br=2, Bc=2, seed=4), prob)


def test_invalid_inputs_rejected(pkg):
    u = np.array([0, 5], np.int32)
    v = np.array([0, 1], np.int32)
    r = np.array([1.0, 2.0], np.float32)
    mdl = pkg.Model(5, 4, 8)
    with pytest.raises(pkg.HccmfError) as e:
        mdl.load(u, v, r)
    assert e.value.code == pkg.ERANGE
    with pytest.raises(pkg.HccmfError):
        mdl.load(np.array([0], np.int32), np.array([0], np.int32), np.array([np.nan], np.float32))
    with pytest.raises(pkg.HccmfError) as e:
        mdl.train_epoch("det")
    assert e.value.code == pkg.ESTATE
    mdl.load(np.array([0, 1], np.int32), np.array([0, 1], np.int32), r)
    mdl.partition(1, (2, 3))
    mdl.init(1)
    with pytest.raises(pkg.HccmfError) as e:
        mdl.train_epoch("det")  # DET needs a square grid
    assert e.value.code == pkg.EINVAL


# ------------------------------------------------------------ a0, a8
def test_init_matches_oracle(pkg, orc):
    for k in (4, 16, 128):
        m, n = 300, 170
        u, v, r = synth.tiny(m, n, 100, seed=k)
        prob = orc.Problem(m, n, k, 0.01, 0.01, u, v, r, seed=77)
        prob.init(123)
        mdl = _gpu_problem(pkg, m, n, k, 0.01, 0.01, u, v, r, seed=77)
        mdl.init(123)
        P, Q = mdl.factors()
        Po, Qo = prob.factors()
        np.testing.assert_allclose(P, Po, rtol=1.2e-7, atol=0)
        np.testing.assert_allclose(Q, Qo, rtol=1.2e-7, atol=0)


@pytest.mark.parametrize("k", [4, 12, 16, 32, 64, 128, 160, 512])
def test_rmse_matches_oracle(pkg, orc, k):
    m, n = 400, 300
    (u, v, r), (tu, tv, tr) = synth.planted(m, n, 8000, 3000, seed=k)
    prob = orc.Problem(m, n, k, 0.01, 0.01, u, v, r, seed=3)
    prob.init(5)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, m, n, k, 0.01, 0.01, u, v, r, seed=3)
    mdl.set_factors(P0, Q0)
    assert mdl.rmse(tu, tv, tr) == pytest.approx(prob.rmse(tu, tv, tr), rel=1e-6)
    # deterministic: same bits twice
    assert mdl.rmse(tu, tv, tr) == mdl.rmse(tu, tv, tr)
    Pg, Qg = mdl.factors()
    assert np.array_equal(Pg, P0) and np.array_equal(Qg, Q0)


# --------------------------------------------------- a5 deterministic epoch
@pytest.mark.parametrize("k,B,gamma,epochs", [(16, 32, 0.05, 1), (16, 32, 0.005, 5), (4, 7, 0.05, 1),
                                               (12, 5, 0.05, 1), (32, 16, 0.02, 2), (48, 9, 0.02, 1),
                                               (64, 16, 0.02, 1), (128, 16, 0.01, 1), (160, 6, 0.01, 1),
                                               (256, 8, 0.005, 1), (512, 4, 0.002, 1)])
def test_det_epoch_parity(pkg, orc, k, B, gamma, epochs):
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=11)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=11)
    mdl.set_factors(P0, Q0)
    for _ in range(epochs):
        mdl.train_epoch("det", "none")
        prob.epoch("det", "none")
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    err = max(np.abs(P - Po).max(), np.abs(Q - Qo).max())
    assert err <= 1e-4, err
    assert mdl.rmse(tu, tv, tr) == pytest.approx(prob.rmse(tu, tv, tr), abs=1e-5)


@pytest.mark.parametrize("sync,G,Br,Bc", [("ring", 2, 4, 8), ("ring", 3, 3, 9), ("allreduce", 2, 4, 4),
                                          ("allreduce", 4, 3, 3)])
def test_det_logical_shards_parity(pkg, orc, sync, G, Br, Bc):
    # T4-i: G logical shards on one device run exactly the multi-GPU schedule
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    k, gamma = 16, 0.05
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
    prob.init(8)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
    _check_partition(mdl, prob)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("det", sync)
        prob.epoch("det", sync)
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4


# ------------------------------------------------------- a6 Hogwild
@pytest.mark.parametrize("atomic", [0, 1])
@pytest.mark.parametrize("k,task,depth,dup", [(128, 64, 1, False), (256, 64, 1, False), (128, 1000, 1, False),
                                              (128, 1000, 2, False), (128, 100, 3, False), (128, 1000, 4, False),
                                              (128, 300, 1, True), (256, 300, 1, True), (128, 300, 2, True),
                                              (128, 300, 4, True),
                                              # k = 32 / 64: the one-rating-per-warp narrow kernel
                                              (32, 64, 0, False), (32, 1000, 1, False), (64, 1000, 3, False),
                                              (32, 300, 2, True), (64, 300, 0, True), (32, 300, 4, True)])
def test_hogwild_single_group_is_the_serial_oracle(pkg, orc, atomic, k, task, depth, dup):
    # One warp = one rating group (k = 32, 64 and k >= 128) walks the tasks in record order: the
    # Hogwild kernel then IS the oracle's serial epoch (task builder, user runs,
    # p_u carry, q forwarding and same-thread red->load ordering all pinned).
    # dup: every rating twice (adjacent after the sort): q forwarding on every other step.
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    if dup:
        u, v, r = (np.concatenate([x, x]) for x in (u, v, r))
    prob = orc.Problem(cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=1, Bc=1, seed=3)
    prob.init(4)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(cfg.m, cfg.n, k, 0.02, cfg.lam)
    mdl.set_option("task_ratings", task)  # > 64: the record ring wraps inside a task
    mdl.set_option("prefetch_depth", depth)
    mdl.set_option("heavy_first", -1)  # record order = the oracle's serial order
    mdl.load(u, v, r)
    mdl.partition(1, (1, 1), seed=3)
    mdl.set_option("hogwild_warps", 1)
    mdl.set_option("vec", k // 128)  # 32 lanes per rating: one group in the one warp
    mdl.set_option("hogwild_atomic", atomic)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("hogwild", "none")
        prob.epoch("serial", "none")
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4


@pytest.mark.parametrize("Bc,scale", [(2, 1.0), (3, 1.0), (8, 1.0), (8, 20.0), (5, 20.0)])
def test_hogwild_single_group_column_phases(pkg, orc, Bc, scale):
    # grid (1, Bc): one launch per column-block phase (C4's configuration); one warp walks every
    # phase's tasks in record order, so the epoch IS the oracle's serial run of the sorted
    # records (blocks (0, 0), (0, 1), ..).  scale 20: ratings on C4's 0..100 range.
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    r = (r * scale).astype(np.float32)
    prob = orc.Problem(cfg.m, cfg.n, 128, 0.005, 1.0, u, v, r, G=1, Br=1, Bc=Bc, seed=3)
    prob.init(4)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(cfg.m, cfg.n, 128, 0.005, 1.0)
    mdl.set_option("heavy_first", -1)
    mdl.load(u, v, r)
    mdl.partition(1, (1, Bc), seed=3)
    mdl.set_option("hogwild_warps", 1)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("hogwild", "none")
        prob.epoch("serial", "none")
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert np.isfinite(P).all() and np.isfinite(Q).all()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4 * max(1.0, scale)


@pytest.mark.parametrize("m,n,nnz,Bc", [(40, 7, 300, 12), (300, 5, 2500, 9), (30, 64, 0, 4), (1, 50, 200, 70)])
def test_hogwild_single_group_empty_blocks(pkg, orc, m, n, nnz, Bc):
    # grid (1, Bc) with empty column blocks (Bc > items, or no ratings at all): the per-block
    # task offsets and the plan's task lists are built on the device (no host copy of the
    # tasks); one warp walks them in record order = the oracle's serial epoch, 1e-4
    u, v, r = synth.tiny(m, n, nnz, seed=m + n + Bc)
    prob = orc.Problem(m, n, 128, 0.02, 0.01, u, v, r, G=1, Br=1, Bc=Bc, seed=7)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(m, n, 128, 0.02, 0.01)
    mdl.set_option("heavy_first", -1)
    mdl.set_option("task_ratings", 7)  # several tasks per block
    mdl.load(u, v, r)
    mdl.partition(1, (1, Bc), seed=7)
    mdl.set_option("hogwild_warps", 1)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("hogwild", "none")
        prob.epoch("serial", "none")
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    mdl.close()
    assert max(np.abs(P - Po).max(initial=0.0), np.abs(Q - Qo).max(initial=0.0)) <= 1e-4


def _band(pkg, orc, cfg_name, frac, k, epochs, sync="none", G=1, Br=1, Bc=1, repeats=2, gamma=None):
    """GPU and oracle test-RMSE curves (same data, same schedule, init seed 1), checked with the
    shared bar of tests/bands.py (R15, R29) for every repeat."""
    cfg = synth.CONFIGS[cfg_name]
    if frac != 1.0:
        cfg = synth.scaled(cfg, frac)
    gamma = cfg.gamma if gamma is None else gamma
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=cfg.seed)
    prob.init(1)
    want = [prob.rmse(tu, tv, tr)]
    for _ in range(epochs):
        prob.epoch("serial", sync)
        want.append(prob.rmse(tu, tv, tr))
    for rep in range(repeats):
        mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=cfg.seed)
        mdl.init(1)
        got = [mdl.rmse(tu, tv, tr)]
        for _ in range(epochs):
            mdl.train_epoch("hogwild", sync)
            got.append(mdl.rmse(tu, tv, tr))
        mdl.close()
        bands.check(got, want, f"{cfg_name} frac={frac} k={k} sync={sync} G={G} grid={Br}x{Bc} rep={rep}",
                    scale=25.0 if cfg.scale == "100" else 1.0)


def test_hogwild_band_c1(pkg, orc):
    # BASELINE.json config 1: 5 epochs, 1 GPU vs the CPU oracle
    _band(pkg, orc, "c1", 1.0, 16, 5, repeats=3)


def test_hogwild_band_c2_full(pkg, orc):
    # BASELINE.json config 2 at full size; band read at E = 20 epochs (R15)
    _band(pkg, orc, "c2", 1.0, 32, 20, repeats=3)  # Hogwild bands run 3 times


@pytest.mark.parametrize("Bc", [1, 4])
def test_hogwild_band_c4_scaled(pkg, orc, Bc):
    # C4's rating scale (0..100, lambda 1) at 5 % size (12.6 M ratings, 31 K items): at the full
    # resident concurrency (4,736 warps, 6.6 items per warp) this diverged to NaN in epoch 1;
    # the staleness budget (R32) sizes the concurrency from gamma (r_rms + lambda) and holds the band
    # (0.005 per 4 rating units: 0.125 on C4's 0..100 range, R29)
    _band(pkg, orc, "c4", 0.05, 128, 5, Bc=Bc, repeats=2)


@pytest.mark.parametrize("sync,G,Bc", [("ring", 4, 4), ("ring", 2, 8), ("allreduce", 2, 1)])
def test_hogwild_logical_shards_band_c2(pkg, orc, sync, G, Bc):
    # multi-GPU schedules on G logical shards; the oracle runs the same schedule serially
    _band(pkg, orc, "c2", 1.0, 32, 20, sync=sync, G=G, Br=1, Bc=Bc, repeats=1)


@pytest.mark.parametrize("k,B,dup", [(128, 24, False), (256, 9, False), (128, 37, True), (512, 12, True),
                                     (512, 5, True)])  # k=512, B=5: slab too big -> register wavefront
def test_det_wavefront_equals_strata(pkg, orc, k, B, dup):
    # the wavefront kernels (Q slab in shared memory: det_wave 1; registers only: 2) and
    # the per-stratum launches (0) apply the same updates in the same per-row /
    # per-column order: bit-identical factors, and the oracle to 1e-4.  dup: every
    # rating duplicated (serial read-after-write of q_v through the slab)
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    if dup:
        u, v, r = (np.concatenate([x[:20000], x[:20000]]) for x in (u, v, r))
    prob = orc.Problem(cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    outs = []
    for wave in (1, 2, 0):
        mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6)
        mdl.set_option("det_wave", wave)
        mdl.set_factors(P0, Q0)
        for _ in range(2):
            mdl.train_epoch("det", "none")
        outs.append(mdl.factors())
    for _ in range(2):
        prob.epoch("det", "none")
    for o in outs[1:]:
        assert np.array_equal(outs[0][0], o[0]) and np.array_equal(outs[0][1], o[1])
    Po, Qo = prob.factors()
    assert max(np.abs(outs[0][0] - Po).max(), np.abs(outs[0][1] - Qo).max()) <= 1e-4


def test_partition_col_balance_bitexact(pkg, orc):
    # R30: the degree-balanced column permutation (host least-loaded placement from the GPU
    # item histogram) and the resulting blocks equal the oracle's bit for bit
    rng = np.random.default_rng(17)
    for trial in range(60):
        m, n = int(rng.integers(1, 15)), int(rng.integers(1, 15))
        nnz = int(rng.integers(0, 120))
        G = int(rng.integers(1, min(m, 3) + 1))
        Br, Bc = int(rng.integers(1, 5)), int(rng.integers(1, 6))
        u, v, r = synth.tiny(m, n, nnz, seed=trial)
        prob = orc.Problem(m, n, 4, 0.01, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=trial % 3, col_balance=1)
        mdl = _gpu_problem(pkg, m, n, 4, 0.01, 0.01, u, v, r, G=G, Br=Br, Bc=Bc, seed=trial % 3, col_balance=True)
        _check_partition(mdl, prob)
        mdl.close()
    cfg = synth.scaled(synth.CONFIGS["c2"], 0.05)
    (u, v, r), _ = synth.make(cfg)
    for G, Br, Bc in [(1, 16, 16), (2, 4, 8), (1, 1, 37)]:
        prob = orc.Problem(cfg.m, cfg.n, 32, cfg.gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5, col_balance=1)
        mdl = _gpu_problem(pkg, cfg.m, cfg.n, 32, cfg.gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5,
                           col_balance=True)
        _check_partition(mdl, prob)
        mdl.close()


@pytest.mark.parametrize("wave,B", [(1, 8), (1, 24), (0, 8), (3, 12)])
def test_det_epoch_parity_col_balance(pkg, orc, wave, B):
    # the DET order on degree-balanced column blocks (R30): every wavefront / the strata
    # against the oracle's serial run of the same partition, 1e-4
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    rng = np.random.default_rng(B)
    v = (rng.zipf(1.4, len(u)) % cfg.n).astype(np.int32)  # skewed items: balancing moves them
    prob = orc.Problem(cfg.m, cfg.n, 128, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6, col_balance=1)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, 128, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6, col_balance=True)
    _check_partition(mdl, prob)
    mdl.set_option("det_wave", wave)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("det", "none")
        prob.epoch("det", "none")
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4


@pytest.mark.parametrize("k,B,skew,dup", [(128, 8, False, False), (128, 8, True, True), (128, 24, True, False),
                                           (256, 12, True, True), (128, 37, False, True), (128, 3, True, False)])
def test_det_chain_wavefront_parity(pkg, orc, k, B, skew, dup):
    # det_wave 3: the chain-parallel wavefront (detchain.cu) keeps every P row's and Q row's
    # update sequence of the DET order (R19) while 4 lane groups walk different item chains
    # of a block: the oracle to 1e-4, deterministic (two runs bit-identical), one launch per
    # epoch once the schedule is built.  skew: Zipf items (long chains, many users shared by
    # several chains of a block: cross-group waits); dup: duplicated cells; B = 8 blocks
    # hold ~125 users each (several shared-memory segments per block).
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    if skew:
        rng = np.random.default_rng(B)
        v = (rng.zipf(1.4, len(u)) % cfg.n).astype(np.int32)
    if dup:
        u, v, r = (np.concatenate([x[:30000], x[:15000]]) for x in (u, v, r))
    prob = orc.Problem(cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    outs = []
    for rep in range(2):
        mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=6)
        mdl.set_option("det_wave", 3)
        mdl.set_factors(P0, Q0)
        mdl.train_epoch("det", "none")  # builds the chain schedule
        assert mdl.info()["det_path"] == (3 if -(-cfg.n // B) <= 64 else 1)  # wmax > 64: the slab wavefront
        l0 = pkg.kernel_launches()
        mdl.train_epoch("det", "none")
        assert pkg.kernel_launches() - l0 == 1
        outs.append(mdl.factors())
        mdl.close()
    for _ in range(2):
        prob.epoch("det", "none")
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    Po, Qo = prob.factors()
    assert max(np.abs(outs[0][0] - Po).max(), np.abs(outs[0][1] - Qo).max()) <= 1e-4


@pytest.mark.parametrize("m,n,nnz,B", [(50, 20, 3000, 37), (40, 300, 4000, 2), (300, 7, 2500, 5), (1, 9, 40, 3),
                                       (9, 1, 40, 4), (30, 30, 0, 6)])
def test_det_chain_wavefront_degenerate_grids(pkg, orc, m, n, nnz, B):
    u, v, r = synth.tiny(m, n, nnz, seed=m + n + B)
    prob = orc.Problem(m, n, 128, 0.02, 0.01, u, v, r, G=1, Br=B, Bc=B, seed=9)
    prob.init(5)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, m, n, 128, 0.02, 0.01, u, v, r, G=1, Br=B, Bc=B, seed=9)
    mdl.set_option("det_wave", 3)
    mdl.set_factors(P0, Q0)
    mdl.train_epoch("det", "none")
    P, Q = mdl.factors()
    mdl.close()
    prob.epoch("det", "none")
    Po, Qo = prob.factors()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4


def test_column_grid_is_the_transposed_row_grid(pkg, orc):
    # f3 / L881-L886: a column grid = the row grid of R^T with P and Q swapped;
    # only P would move between shards ("transmitting P only", L1216-L1218)
    m, n, k, B, G = 300, 700, 16, 4, 2
    (u, v, r), (tu, tv, tr) = synth.planted(m, n, 20000, 2000, seed=4)
    rng = np.random.default_rng(1)
    P0 = rng.uniform(0, 0.3, (m, k)).astype(np.float32)
    Q0 = rng.uniform(0, 0.3, (n, k)).astype(np.float32)
    prob = orc.Problem(n, m, k, 0.05, 0.01, v, u, r, G=G, Br=B, Bc=G * B, seed=8)  # R^T
    prob.set_factors(Q0, P0)
    mdl = pkg.Model(m, n, k, 0.05, 0.01)
    mdl.load(u, v, r)
    mdl.partition(G, (B, G * B), seed=8, grid_dim="cols")
    assert mdl.info()["transposed"] == 1 and mdl.info()["m"] == n
    _check_partition(mdl, prob)
    mdl.set_factors(P0, Q0)
    assert mdl.rmse(tu, tv, tr) == pytest.approx(prob.rmse(tv, tu, tr), rel=1e-6)
    for _ in range(2):
        mdl.train_epoch("det", "ring")
        prob.epoch("det", "ring")
    P, Q = mdl.factors()
    Qo, Po = prob.factors()
    assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4
    # the paper's rule picks columns here (n > m); init is orientation-independent
    a = pkg.Model(m, n, k)
    a.load(u, v, r)
    a.partition(1, (1, 1), seed=8, grid_dim="auto")
    assert a.info()["transposed"] == 1
    a.init(9)
    b = pkg.Model(m, n, k)
    b.load(u, v, r)
    b.partition(1, (1, 1), seed=8, grid_dim="rows")
    b.init(9)
    (Pa, Qa), (Pb, Qb) = a.factors(), b.factors()
    assert np.array_equal(Pa, Pb) and np.array_equal(Qa, Qb)


@pytest.mark.parametrize("phases", [2, 4])
def test_hogwild_allreduce_sub_epoch_sync_band_c2(pkg, orc, phases):
    # R22 / SURVEY f4: all-reduce with `phases` rounds per epoch vs the oracle's
    # phased replica schedule (serial inside each replica), 20 epochs, C2 full size
    cfg = synth.CONFIGS["c2"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    G, Br = 2, 4
    prob = orc.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=1, seed=cfg.seed)
    prob.init(1)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=1, seed=cfg.seed)
    mdl.set_option("sync_phases", phases)
    mdl.init(1)
    want, got = [prob.rmse(tu, tv, tr)], [mdl.rmse(tu, tv, tr)]
    for _ in range(20):
        prob.epoch_phased(phases)
        mdl.train_epoch("hogwild", "allreduce")
        want.append(prob.rmse(tu, tv, tr))
        got.append(mdl.rmse(tu, tv, tr))
    bands.check(got, want, f"c2 allreduce phases={phases}")


def test_distributed_handle_world1_matches_single(pkg, orc):
    # the NCCL backend's bootstrap on one rank: the unique id travels through
    # torch.distributed and ncclCommInitRank builds a one-rank communicator.  With world = 1
    # and G = 1 no collective runs (every data-plane call site is guarded by world > 1 and
    # the epochs degenerate to SYNC_NONE), so this pins the handle plumbing only: results
    # equal the single-process handle bit for bit.  The multi-rank data plane itself runs in
    # tests/test_gpu_loopback.py (every call site, G = 2..8 ranks on one GPU).
    import os
    import socket
    import torch.distributed as dist
    sock = socket.socket()
    sock.bind(("127.0.0.1", 0))
    port = sock.getsockname()[1]
    sock.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        cfg = synth.CONFIGS["c1"]
        (u, v, r), (tu, tv, tr) = synth.make(cfg)
        outs = []
        for distributed in (True, False):
            mdl = pkg.Model(cfg.m, cfg.n, 128, 0.02, cfg.lam, dist=distributed, device=0)
            mdl.load(u, v, r)
            mdl.partition(1, (8, 8), seed=4)
            mdl.init(3)
            mdl.set_option("hogwild_warps", 1)  # k = 128: one group in one warp, deterministic
            for sched, sync in (("det", "none"), ("det", "allreduce"), ("hogwild", "ring")):
                mdl.train_epoch(sched, sync)
            outs.append((mdl.factors(), mdl.rmse(tu, tv, tr), mdl.info()["world"]))
            mdl.close()
        (Pd, Qd), rd, wd = outs[0]
        (Ps, Qs), rs, ws = outs[1]
        assert wd == 1 and ws == 1
        assert np.array_equal(Pd, Ps) and np.array_equal(Qd, Qs) and rd == rs
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("sync,G,Br,Bc", [("ring", 2, 4, 8), ("ring", 3, 3, 9), ("allreduce", 2, 4, 4)])
def test_det_wire_fp16_logical_shards(pkg, orc, sync, G, Br, Bc):
    # Strategy 2 (L1234-L1249, R25): Q crosses every shard boundary as binary16.
    # Bar: the fp32-vs-fp64 1e-4 plus one binary16 rounding flip (2^-10 |x|) where the
    # two sides' values straddle a binary16 rounding boundary.
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    k, gamma = 16, 0.05
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
    prob.init(8)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
    mdl.set_option("wire_fp16", 1)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("det", sync)
        prob.epoch_wire16("det", sync)
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert np.all(np.abs(Q - Qo) <= 1e-4 + 2.0 ** -10 * np.abs(Qo))
    assert np.all(np.abs(P - Po) <= 1e-4 + 2.0 ** -10 * np.abs(Po))
    # every Q value left the last transfer as a binary16 number
    assert np.array_equal(Q.astype(np.float16).astype(np.float32), Q)


def test_hogwild_ring_wire_fp16_band_c2(pkg, orc):
    # the paper's claim that FP16 transmission does not cost accuracy, on C2 at 20 epochs
    cfg = synth.CONFIGS["c2"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    G, Bc = 4, 8
    prob = orc.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=1, Bc=Bc, seed=cfg.seed)
    prob.init(1)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=1, Bc=Bc, seed=cfg.seed)
    mdl.set_option("wire_fp16", 1)
    mdl.init(1)
    want, got = [prob.rmse(tu, tv, tr)], [mdl.rmse(tu, tv, tr)]
    for _ in range(20):
        prob.epoch_wire16("serial", "ring")
        mdl.train_epoch("hogwild", "ring")
        want.append(prob.rmse(tu, tv, tr))
        got.append(mdl.rmse(tu, tv, tr))
    bands.check(got, want, "c2 ring G=4 Bc=8 wire16 (logical)")


# ---------------------------------------- binary16 storage of Q (f1, R26)
# Both sides round every q_v write to binary16, but the CUDA kernel rounds its fp32
# result while the oracle rounds its fp64 result; where the two straddle a rounding
# boundary the stored q differs by one binary16 ulp (2^-10 |x| at most).  Bar: see
# _check_q16 (R26).
def _q16_bar(x, ulps=2):
    return 1e-4 + np.abs(x) * ulps * 2.0 ** -10


def _check_q16(P, Po, Q, Qo):
    # Each flip (a rounding boundary between the fp32 and the fp64 result) is one ulp in one
    # element; it is carried into the next updates of that item and of the users that
    # meet it, where it can cause further flips.  Bar: every element within 8 binary16
    # ulps, and at most 0.1 % of them beyond 2 ulps.
    for a, b in ((P, Po), (Q, Qo)):
        d = np.abs(a - b)
        assert np.all(d <= _q16_bar(b, 8)), d.max()
        assert np.mean(d > _q16_bar(b, 2)) <= 1e-3, np.mean(d > _q16_bar(b, 2))


@pytest.mark.parametrize("k,B,epochs,sr", [(128, 8, 1, False), (128, 8, 3, False), (256, 4, 1, False),
                                           (128, 8, 1, True), (128, 8, 3, True), (256, 4, 2, True)])
def test_det_epoch_parity_q16(pkg, orc, k, B, epochs, sr):
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    gamma = 0.02
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=11)
    prob.init(2)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(cfg.m, cfg.n, k, gamma, cfg.lam)
    mdl.load(u, v, r)
    mdl.partition(1, (B, B), seed=11, storage="fp16sr" if sr else "fp16")
    mdl.set_factors(P0, Q0)
    for t in range(epochs):  # SR: the random words of epoch t (R27) are the same on both sides
        mdl.train_epoch("det", "none")
        prob.epoch_q16("det", "none", sr=sr, t=t)
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    assert np.array_equal(Q.astype(np.float16).astype(np.float32), Q)  # Q holds binary16 values
    _check_q16(P, Po, Q, Qo)
    assert mdl.rmse(tu, tv, tr) == pytest.approx(prob.rmse(tu, tv, tr), abs=1e-4)


@pytest.mark.parametrize("atomic,sr,dup", [(0, False, False), (1, False, False), (0, True, False), (1, True, False),
                                           (0, False, True), (1, False, True), (0, True, True), (1, True, True)])
def test_hogwild_single_group_q16(pkg, orc, atomic, sr, dup):
    # one warp walks the tasks in record order: the binary16 Hogwild kernel is then the
    # oracle's serial epoch with binary16 Q (atomic: the increment is itself rounded
    # to binary16 before the add, one more rounding than the oracle's).  dup: every
    # rating twice, so every other rating repeats the previous item (q forwarding)
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    if dup:
        u, v, r = (np.concatenate([x, x]) for x in (u, v, r))
    k = 128
    prob = orc.Problem(cfg.m, cfg.n, k, 0.02, cfg.lam, u, v, r, G=1, Br=1, Bc=1, seed=3)
    prob.init(4)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(cfg.m, cfg.n, k, 0.02, cfg.lam)
    mdl.set_option("task_ratings", 300)
    mdl.set_option("heavy_first", -1)
    mdl.load(u, v, r)
    mdl.partition(1, (1, 1), seed=3, storage="fp16sr" if sr else "fp16")
    mdl.set_option("hogwild_warps", 1)
    mdl.set_option("hogwild_atomic", atomic)
    mdl.set_factors(P0, Q0)
    for t in range(2):  # SR: serially, the atomic add of (SR(q + dq) - q) stores SR(q + dq)
        mdl.train_epoch("hogwild", "none")
        prob.epoch_q16("serial", "none", add16=bool(atomic) and not sr, sr=sr, t=t)
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    _check_q16(P, Po, Q, Qo)


@pytest.mark.parametrize("sync,G,Br,Bc,sr", [("ring", 2, 4, 8, False), ("allreduce", 2, 4, 4, False),
                                             ("ring", 2, 4, 8, True), ("allreduce", 2, 4, 4, True)])
def test_det_logical_shards_parity_q16(pkg, orc, sync, G, Br, Bc, sr):
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    k, gamma = 128, 0.02
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=5)
    prob.init(8)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    mdl = pkg.Model(cfg.m, cfg.n, k, gamma, cfg.lam)
    mdl.load(u, v, r)
    mdl.partition(G, (Br, Bc), seed=5, storage="fp16sr" if sr else "fp16")
    mdl.set_factors(P0, Q0)
    for t in range(2):
        mdl.train_epoch("det", sync)
        prob.epoch_q16("det", sync, sr=sr, t=t)
    P, Q = mdl.factors()
    Po, Qo = prob.factors()
    _check_q16(P, Po, Q, Qo)


def test_q16_storage_rejects_unsupported_geometry(pkg):
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    mdl = pkg.Model(cfg.m, cfg.n, 16, cfg.gamma, cfg.lam)
    mdl.load(u, v, r)
    mdl.partition(1, (1, 1), seed=1, storage="fp16")
    mdl.init(1)
    with pytest.raises(pkg.HccmfError) as ei:
        mdl.train_epoch("hogwild", "none")
    assert ei.value.code == pkg.EINVAL


def test_kernel_launch_counter(pkg):
    # hccmf_kernel_launches counts what the library launched (bench.py's gpu_launches):
    # a single-shard DET epoch on a square grid is ONE wavefront kernel, a Hogwild epoch on
    # a 1 x Bc grid one SGD launch per column block, an RMSE evaluation three kernels
    # (validation of the test ratings, per-block partial sums, the fixed-order final sum)
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, 128, 0.01, cfg.lam, u, v, r, G=1, Br=8, Bc=8, seed=3)
    mdl.init(1)
    l0 = pkg.kernel_launches()
    mdl.train_epoch("det", "none")
    assert pkg.kernel_launches() - l0 == 1
    l0 = pkg.kernel_launches()
    mdl.rmse(tu, tv, tr)
    assert pkg.kernel_launches() - l0 == 3
    mdl.close()
    mdl = _gpu_problem(pkg, cfg.m, cfg.n, 128, 0.01, cfg.lam, u, v, r, G=1, Br=1, Bc=4, seed=3)
    mdl.init(1)
    mdl.train_epoch("hogwild", "none")  # builds the plan
    l0 = pkg.kernel_launches()
    mdl.train_epoch("hogwild", "none")
    assert pkg.kernel_launches() - l0 == 4
    mdl.close()


@pytest.mark.parametrize("m,n,nnz,B,k", [(50, 20, 3000, 37, 128), (40, 300, 4000, 2, 128), (300, 7, 2500, 5, 256),
                                         (64, 64, 0, 8, 128), (1, 90, 400, 3, 128)])
def test_det_wavefront_degenerate_grids(pkg, orc, m, n, nnz, B, k):
    # the slab wavefront on degenerate geometries: more column blocks than items (empty,
    # zero-width slabs), more row blocks than rows, one row, an empty problem, duplicated
    # cells (synth.tiny): one launch, bit-identical to the per-stratum launches, oracle to 1e-4
    u, v, r = synth.tiny(m, n, nnz, seed=m + n + B)
    prob = orc.Problem(m, n, k, 0.02, 0.01, u, v, r, G=1, Br=B, Bc=B, seed=9)
    prob.init(5)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    outs = []
    for wave in (1, 0):
        mdl = _gpu_problem(pkg, m, n, k, 0.02, 0.01, u, v, r, G=1, Br=B, Bc=B, seed=9)
        mdl.set_option("det_wave", wave)
        mdl.set_factors(P0, Q0)
        l0 = pkg.kernel_launches()
        mdl.train_epoch("det", "none")
        if wave == 1:
            assert pkg.kernel_launches() - l0 == 1
        outs.append(mdl.factors())
        mdl.close()
    prob.epoch("det", "none")
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    Po, Qo = prob.factors()
    assert max(np.abs(outs[0][0] - Po).max(), np.abs(outs[0][1] - Qo).max()) <= 1e-4


@pytest.mark.parametrize("Bc", [1, 3])
def test_probe_roundtrip_leaves_the_model_alone(pkg, Bc):
    # the in-run ceiling probes (bench.py binding_frac): every mode returns a positive time, on a
    # (1, Bc) grid phase by phase, and none of them changes the model's factors (the reductions go
    # to a scratch Q; the p_u stream mode stores back the rows it loaded)
    cfg = synth.CONFIGS["c1"]
    (u, v, r), _ = synth.make(cfg)
    mdl = pkg.Model(cfg.m, cfg.n, 128, 0.005, 0.01)
    mdl.load(u, v, r)
    mdl.partition(1, (1, Bc), seed=2)
    mdl.init(3)
    P0, Q0 = mdl.factors()
    for mode in ("red_f32", "ldred_f16", "ldred_f32", "q_stream", "p_stream", "bulkred_f32", "bulkldred_f32",
                 "ldbulkred_f32"):
        assert mdl.probe_roundtrip(mode, reps=1) > 0.0, mode
    P1, Q1 = mdl.factors()
    mdl.close()
    assert np.array_equal(P0, P1) and np.array_equal(Q0, Q1)
