"""The multi-rank data plane (row a7) executed on ONE GPU through the loopback
communicator (hccmf_create_loopback): G handles, one host thread each, exchanging Q with the
same call sites, buffers and stream/event ordering as G NCCL ranks.

Every call site of the data plane runs here -- the stage-wise ring, the pipelined per-column-
block ring on its comm stream, binary16 ring transfers, the ring-group broadcasts that
materialise Q, the fp32 Q average, the binary16 Q average (all-to-all + fp64 mean + all-gather),
the RMSE reduction, the P export, and the three steps of sliced ingest -- and is checked
against the oracle's serialisation of the same schedule (R19):
  * DET ring / all-reduce: max-abs <= 1e-4 vs the oracle;
  * binary16 wire (Strategy 2, L1234-L1249, R25): 1e-4 + one binary16 flip vs orc_epoch_wire16;
  * Hogwild pipelined ring (L1251-L1269): test RMSE within 0.005 of the oracle's ring order,
    3 runs, full-size C2, each rank launching its own column blocks (one rank's real race);
  * sliced ingest: the per-rank partitions concatenate to the single-process partition, bit
    for bit (L543-L548).
"""
import threading

import numpy as np
import pytest

import bands
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


def run_ranks(pkg, G, m, n, k, gamma, lam, body, timeout=900):
    """body(rank, model) on G loopback handles, one thread each; returns the G results."""
    hub = pkg.Hub(G)
    out, errs = [None] * G, [None] * G

    def work(r):
        try:
            mdl = pkg.Model(m, n, k, gamma, lam, hub=hub, rank=r, device=0)
            try:
                out[r] = body(r, mdl)
            finally:
                mdl.close()
        except BaseException as e:  # noqa: BLE001 -- re-raised below
            errs[r] = e

    ts = [threading.Thread(target=work, args=(r,), daemon=True) for r in range(G)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout)
    hub.close()
    assert not any(t.is_alive() for t in ts), "a loopback rank hung"
    for e in errs:
        if e is not None:
            raise e
    return out


def _c1(k=16, gamma=0.05):
    cfg = synth.CONFIGS["c1"]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    return cfg, (u, v, r), (tu, tv, tr), k, gamma


def _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, seed):
    prob = orc.Problem(cfg.m, cfg.n, k, gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=seed)
    prob.init(8)
    P0, Q0 = [x.astype(np.float32) for x in prob.factors()]
    prob.set_factors(P0, Q0)
    return prob, P0, Q0


@pytest.mark.parametrize("sync,G,Br,Bc", [("ring", 2, 4, 8), ("ring", 3, 3, 9), ("ring", 4, 2, 8),
                                          ("allreduce", 2, 4, 4), ("allreduce", 4, 3, 3)])
def test_loopback_det_parity(pkg, orc, sync, G, Br, Bc):
    cfg, (u, v, r), (tu, tv, tr), k, gamma = _c1()
    prob, P0, Q0 = _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, 5)

    def body(rank, mdl):
        mdl.load(u, v, r)
        mdl.partition(G, (Br, Bc), seed=5)
        inf = mdl.info()
        assert inf["world"] == G and inf["shard_lo"] == rank and inf["shard_hi"] == rank + 1
        recs = mdl.records()
        mdl.set_factors(P0, Q0)
        for _ in range(2):
            mdl.train_epoch("det", sync)
        P, Q = mdl.factors()
        return recs, inf, P, Q, mdl.rmse(tu, tv, tr), mdl.comm_counts()

    res = run_ranks(pkg, G, cfg.m, cfg.n, k, gamma, cfg.lam, body)
    for _ in range(2):
        prob.epoch("det", sync)
    Po, Qo = prob.factors()
    want_rmse = prob.rmse(tu, tv, tr)
    bps = Br * Bc
    for rank, ((gu, gv, gr), inf, P, Q, rm, cc) in enumerate(res):
        a, b = prob.off[rank * bps], prob.off[(rank + 1) * bps]
        assert np.array_equal(gu, prob.ru[a:b]) and np.array_equal(gv, prob.rv[a:b])
        assert np.array_equal(gr.view(np.int32), prob.rr[a:b].view(np.int32))
        assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4
        assert rm == pytest.approx(want_rmse, abs=1e-5)
        if sync == "ring":
            assert cc["ring_stage"] == 2 * G and cc["materialize_q"] >= 1
        else:
            assert cc["allreduce_q"] == 2
        assert cc["rmse"] == 1 and cc["export_p"] == 1
    # every rank exports the same matrices
    for r_ in res[1:]:
        assert np.array_equal(r_[2], res[0][2]) and np.array_equal(r_[3], res[0][3])


@pytest.mark.parametrize("sync,G,Br,Bc", [("ring", 2, 4, 8), ("ring", 3, 3, 9), ("allreduce", 2, 4, 4),
                                          ("allreduce", 3, 2, 2)])
def test_loopback_det_equals_logical_shards(pkg, orc, sync, G, Br, Bc):
    # the loopback data plane and the logical-shard backend run the same blocks with the same
    # kernels: DET factors are bit-identical (the all-reduce mean is fp64 in rank order on both)
    cfg, (u, v, r), (tu, tv, tr), k, gamma = _c1()
    _, P0, Q0 = _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, 5)
    mdl = pkg.Model(cfg.m, cfg.n, k, gamma, cfg.lam)
    mdl.load(u, v, r)
    mdl.partition(G, (Br, Bc), seed=5)
    mdl.set_factors(P0, Q0)
    for _ in range(2):
        mdl.train_epoch("det", sync)
    Pl, Ql = mdl.factors()
    rl = mdl.rmse(tu, tv, tr)
    mdl.close()

    def body(rank, m_):
        m_.load(u, v, r)
        m_.partition(G, (Br, Bc), seed=5)
        m_.set_factors(P0, Q0)
        for _ in range(2):
            m_.train_epoch("det", sync)
        P, Q = m_.factors()
        return P, Q, m_.rmse(tu, tv, tr)

    for P, Q, rm in run_ranks(pkg, G, cfg.m, cfg.n, k, gamma, cfg.lam, body):
        assert np.array_equal(P, Pl) and np.array_equal(Q, Ql)
        assert rm == pytest.approx(rl, rel=1e-12)


@pytest.mark.parametrize("sync,G,Br,Bc", [("ring", 2, 4, 8), ("ring", 3, 3, 9), ("allreduce", 2, 4, 4),
                                          ("allreduce", 4, 3, 3)])
def test_loopback_det_wire_fp16(pkg, orc, sync, G, Br, Bc):
    # Strategy 2 on the real data plane: ring groups travel as binary16; the all-reduce ships
    # binary16 chunks, sums the G rounded copies in fp64 and rounds the mean once (R25)
    cfg, (u, v, r), _, k, gamma = _c1()
    prob, P0, Q0 = _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, 5)

    def body(rank, mdl):
        mdl.load(u, v, r)
        mdl.partition(G, (Br, Bc), seed=5)
        mdl.set_option("wire_fp16", 1)
        mdl.set_factors(P0, Q0)
        for _ in range(2):
            mdl.train_epoch("det", sync)
        P, Q = mdl.factors()
        return P, Q, mdl.comm_counts()

    res = run_ranks(pkg, G, cfg.m, cfg.n, k, gamma, cfg.lam, body)
    for _ in range(2):
        prob.epoch_wire16("det", sync)
    Po, Qo = prob.factors()
    for P, Q, cc in res:
        assert np.all(np.abs(Q - Qo) <= 1e-4 + 2.0 ** -10 * np.abs(Qo))
        assert np.all(np.abs(P - Po) <= 1e-4 + 2.0 ** -10 * np.abs(Po))
        assert np.array_equal(Q.astype(np.float16).astype(np.float32), Q)
        if sync == "ring":
            assert cc["ring_wire16"] == 2 * G
        else:
            assert cc["allreduce_q16"] == 2 and cc["allreduce_q"] == 0


def test_loopback_wire16_allreduce_is_one_rounding(pkg, orc):
    # the binary16 all-reduce computes binary16(sum_s binary16(Q_s) / G) with an fp64 sum,
    # not a binary16 reduction with a rounding per hop: compare with the logical backend,
    # which evaluates that definition in one kernel (average_half_kernel) -- bit-identical
    cfg, (u, v, r), _, k, gamma = _c1()
    G, Br, Bc = 4, 3, 3
    _, P0, Q0 = _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, 5)
    mdl = pkg.Model(cfg.m, cfg.n, k, gamma, cfg.lam)
    mdl.load(u, v, r)
    mdl.partition(G, (Br, Bc), seed=5)
    mdl.set_option("wire_fp16", 1)
    mdl.set_factors(P0, Q0)
    mdl.train_epoch("det", "allreduce")
    Pl, Ql = mdl.factors()
    mdl.close()

    def body(rank, m_):
        m_.load(u, v, r)
        m_.partition(G, (Br, Bc), seed=5)
        m_.set_option("wire_fp16", 1)
        m_.set_factors(P0, Q0)
        m_.train_epoch("det", "allreduce")
        return m_.factors()

    for P, Q in run_ranks(pkg, G, cfg.m, cfg.n, k, gamma, cfg.lam, body):
        assert np.array_equal(Q, Ql) and np.array_equal(P, Pl)


@pytest.mark.parametrize("G,Br,Bc,bal", [(2, 4, 8, 0), (3, 5, 7, 0), (4, 8, 32, 0), (4, 1, 4, 0), (3, 2, 6, 1)])
def test_loopback_sliced_ingest_concatenates_to_single_process(pkg, orc, G, Br, Bc, bal):
    # each rank loads 1/G (uneven, one empty) of the COO; the exchange + local sort reproduce the
    # single-process partition: perms, bounds, global block offsets and every shard's records
    cfg = synth.scaled(synth.CONFIGS["c2"], 0.02)
    (u, v, r), _ = synth.make(cfg)
    nnz = len(u)
    cuts = np.sort(np.random.default_rng(G).integers(0, nnz, G - 1))
    cuts[0] = cuts[0] // 3
    edges = [0, *cuts.tolist(), nnz]
    if G >= 3:
        edges[2] = edges[1]  # rank 1 loads nothing
    prob = orc.Problem(cfg.m, cfg.n, 32, cfg.gamma, cfg.lam, u, v, r, G=G, Br=Br, Bc=Bc, seed=9, col_balance=bal)

    def body(rank, mdl):
        a, b = edges[rank], edges[rank + 1]
        mdl.load_slice(u[a:b], v[a:b], r[a:b])
        mdl.partition(G, (Br, Bc), seed=9, col_balance=bool(bal))
        return mdl.get_partition(), mdl.records(), mdl.info(), mdl.comm_counts()

    res = run_ranks(pkg, G, cfg.m, cfg.n, 32, cfg.gamma, cfg.lam, body)
    bps = Br * Bc
    for rank, ((b, off, pr, pc), (gu, gv, gr), inf, cc) in enumerate(res):
        assert np.array_equal(pr, prob.perm_row) and np.array_equal(pc, prob.perm_col)
        assert np.array_equal(b, prob.b) and np.array_equal(off, prob.off)
        lo, hi = prob.off[rank * bps], prob.off[(rank + 1) * bps]
        assert inf["nnz"] == nnz and inf["local_nnz"] == hi - lo
        assert np.array_equal(gu, prob.ru[lo:hi]) and np.array_equal(gv, prob.rv[lo:hi])
        assert np.array_equal(gr.view(np.int32), prob.rr[lo:hi].view(np.int32))
        assert cc["ingest_hist"] == 1 + bal and cc["ingest_exchange"] == 1 and cc["ingest_blocks"] == 1


def test_loopback_sliced_ingest_trains_like_replicated(pkg, orc):
    # a DET ring epoch after sliced ingest equals the oracle (the records each rank trains on
    # are the same bytes as after a replicated load)
    cfg, (u, v, r), (tu, tv, tr), k, gamma = _c1()
    G, Br, Bc = 3, 3, 9
    prob, P0, Q0 = _oracle_start(orc, cfg, k, gamma, u, v, r, G, Br, Bc, 5)
    edges = np.linspace(0, len(u), G + 1).astype(np.int64)

    def body(rank, mdl):
        a, b = edges[rank], edges[rank + 1]
        mdl.load_slice(u[a:b], v[a:b], r[a:b])
        mdl.partition(G, (Br, Bc), seed=5)
        mdl.set_factors(P0, Q0)
        mdl.train_epoch("det", "ring")
        return mdl.factors()

    res = run_ranks(pkg, G, cfg.m, cfg.n, k, gamma, cfg.lam, body)
    prob.epoch("det", "ring")
    Po, Qo = prob.factors()
    for P, Q in res:
        assert max(np.abs(P - Po).max(), np.abs(Q - Qo).max()) <= 1e-4


def test_loopback_every_data_plane_site_runs(pkg, orc):
    # one job that drives every call site of the data plane at least once (comm counters)
    cfg, (u, v, r), (tu, tv, tr), _, _ = _c1()
    k, G = 128, 2
    edges = np.linspace(0, len(u), G + 1).astype(np.int64)

    def body(rank, mdl):
        a, b = edges[rank], edges[rank + 1]
        mdl.load_slice(u[a:b], v[a:b], r[a:b])
        mdl.partition(G, (2, 2 * G), seed=3)
        mdl.init(2)
        mdl.train_epoch("det", "ring")                 # ring_stage + materialize_q (next call)
        mdl.train_epoch("hogwild", "ring")             # ring_block on the comm stream
        mdl.set_option("wire_fp16", 1)
        mdl.train_epoch("hogwild", "ring")             # ring_wire16
        mdl.train_epoch("hogwild", "allreduce")        # allreduce_q16
        mdl.set_option("wire_fp16", 0)
        mdl.train_epoch("hogwild", "allreduce")        # allreduce_q
        rm = mdl.rmse(tu, tv, tr)                      # rmse
        P, Q = mdl.factors()                           # export_p
        return rm, P, Q, mdl.comm_counts()

    res = run_ranks(pkg, G, cfg.m, cfg.n, k, 0.005, cfg.lam, body)
    for rm, P, Q, cc in res:
        assert np.isfinite(rm) and np.isfinite(P).all() and np.isfinite(Q).all()
        missing = [s for s, c in cc.items() if c == 0]
        assert not missing, (missing, cc)
    assert np.array_equal(res[0][1], res[1][1]) and np.array_equal(res[0][2], res[1][2])


def _golden_ring(name, G, Bc):
    """The oracle's ring-order curve stored by tools/oracle_curves.py ring:<name>:G:Bc, or None."""
    import json
    import os
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden",
                        f"oracle_curve_{name}_ring_G{G}_Bc{Bc}.json")
    return json.load(open(path)) if os.path.exists(path) else None


def _hogwild_ring_band(pkg, orc, cfg, G, Bc, epochs, repeats, wire16=False, storage="fp32", seed_init=1,
                       oracle_curve=None):
    """(oracle curve, GPU curves [repeats x (epochs + 1)]); curve[0] is before training."""
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    if oracle_curve is not None:
        curve_o = list(oracle_curve)
    else:
        prob = orc.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=1, Bc=Bc, seed=cfg.seed)
        prob.init(seed_init)
        curve_o = [prob.rmse(tu, tv, tr)]
        for _ in range(epochs):
            if wire16:
                prob.epoch_wire16("serial", "ring")
            else:
                prob.epoch("serial", "ring")
            curve_o.append(prob.rmse(tu, tv, tr))
    edges = np.linspace(0, len(u), G + 1).astype(np.int64)

    def body(rank, mdl):
        a, b = edges[rank], edges[rank + 1]
        mdl.load_slice(u[a:b], v[a:b], r[a:b])
        mdl.partition(G, (1, Bc), seed=cfg.seed, storage=storage)
        mdl.set_option("wire_fp16", int(wire16))
        mdl.init(seed_init)
        curve = [mdl.rmse(tu, tv, tr)]
        for _ in range(epochs):
            mdl.train_epoch("hogwild", "ring")
            curve.append(mdl.rmse(tu, tv, tr))
        return curve, mdl.comm_counts()

    runs = []
    for _ in range(repeats):
        res = run_ranks(pkg, G, cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, body, timeout=3600)
        curve, cc = res[0]
        assert all(x[0] == curve for x in res)  # the RMSE is one all-reduced number
        assert cc["ring_block"] == epochs * Bc
        runs.append(curve)
    return np.array(curve_o), np.array(runs)


@pytest.mark.parametrize("G,Bc", [(2, 2), (4, 4), (8, 8), (4, 8)])
def test_loopback_hogwild_pipelined_ring_band_c2(pkg, orc, G, Bc):
    # full-size C2, 20 epochs (R15), 3 runs: every rank launches its own
    # column blocks with the per-launch concurrency cap (R14, R28), transfers overlap compute
    cfg = synth.CONFIGS["c2"]
    ref = _golden_ring("c2", G, Bc)
    want, runs = _hogwild_ring_band(pkg, orc, cfg, G, Bc, 20, 3, oracle_curve=ref and ref["test_rmse"])
    for i, run in enumerate(runs):
        bands.check(run, want, f"c2 loopback ring G={G} Bc={Bc} run={i}")


@pytest.mark.parametrize("G", [2, 4, 8])
def test_loopback_hogwild_ring_band_c3_full(pkg, orc, G):
    # full-size C3 at one rank's real geometry for G = 2, 4, 8 (bench.py's ring grid: Bc = G),
    # 10 epochs, 3 runs, against the oracle's ring serialisation stored by
    # tools/oracle_curves.py ring:c3:G:G (the CPU oracle takes ~8 min per curve)
    ref = _golden_ring("c3", G, G)
    if ref is None:
        pytest.skip("tools/oracle_curves.py ring:c3:G:G not run")
    cfg = synth.CONFIGS["c3"]
    _, runs = _hogwild_ring_band(pkg, orc, cfg, G, G, ref["epochs"], 3, oracle_curve=ref["test_rmse"])
    for i, run in enumerate(runs):
        bands.check(run, ref["test_rmse"], f"c3 loopback ring G={G} Bc={G} run={i}")


def test_loopback_hogwild_ring_wire16_band_c2(pkg, orc):
    cfg = synth.CONFIGS["c2"]
    want, runs = _hogwild_ring_band(pkg, orc, cfg, 4, 8, 20, 1, wire16=True)
    bands.check(runs[0], want, "c2 loopback ring G=4 Bc=8 wire16")
