"""Multi-process (gloo, CPU) tests of the distributed host logic (-m "not gpu").

Each rank asks libhccmf for the schedule its shard executes (hccmf_schedule: the
same block lists and ring exchange ranges the CUDA runtime uses, no device
needed), runs its blocks with the oracle's serial update, and exchanges Q column
groups with real point-to-point messages over gloo exactly as the NCCL ring does
(send group (s+t) mod G to s-1, receive (s+t+1) mod G from s+1).  The gathered
result must equal the single-process oracle epoch in the canonical ring order
(R19) bit for bit; the all-reduce mode must equal the replica oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _problem(G, Br, Bc):
    import oracle
    import synth
    m, n, k = 40, 30, 8
    u, v, r = synth.tiny(m, n, 600, seed=17)
    prob = oracle.Problem(m, n, k, 0.05, 0.02, u, v, r, G=G, Br=Br, Bc=Bc, seed=9)
    prob.init(3)
    return prob


def _worker(rank, G, Br, Bc, sched, sync, epochs, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=G)
    import oracle
    import paper_conf_icpp_huangylhbl21_b200 as hc
    prob = _problem(G, Br, Bc)
    P, Q = prob.P, prob.Q
    launches, stages, ring = hc.schedule(G, Br, Bc, prob.n, sched, sync, shard=rank)
    for _ in range(epochs):
        Qw = Q.copy() if sync == "allreduce" else Q
        stage = 0

        def exchange(t):
            sl, sh, rl, rh = (int(x) for x in ring[t])
            send = torch.from_numpy(np.ascontiguousarray(Qw[sl:sh]))
            recv = torch.empty((rh - rl, Q.shape[1]), dtype=torch.float64)
            reqs = [dist.isend(send, (rank - 1) % G), dist.irecv(recv, (rank + 1) % G)]
            for q in reqs:
                q.wait()
            Qw[rl:rh] = recv.numpy()

        for blocks, st in zip(launches, stages):
            while sync == "ring" and stage < st:
                exchange(stage)
                stage += 1
            for b in blocks:
                oracle.run(int(prob.off[b]), int(prob.off[b + 1]), prob.k, prob.gamma, prob.lam, prob.ru, prob.rv,
                           prob.rr, P, Qw)
        while sync == "ring" and stage < G:
            exchange(stage)
            stage += 1
        if sync == "allreduce":
            t = torch.from_numpy(Qw)
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
            Q[:] = t.numpy() / G
    # gather: P rows of this shard, Q column group `rank` (ring) or all of Q
    b0, b1 = int(prob.b[rank]), int(prob.b[rank + 1])
    if sync == "ring":
        a0, a1 = hc.schedule(G, Br, Bc, prob.n, sched, sync, shard=rank)[2][0][:2]
        q_part = (int(a0), int(a1), Q[int(a0):int(a1)].copy())
    else:
        q_part = (0, prob.n, Q.copy())
    parts = [None] * G
    dist.all_gather_object(parts, (b0, b1, P[b0:b1].copy(), q_part))
    if rank == 0:
        Pg = np.full_like(P, np.nan)
        Qg = np.full_like(Q, np.nan)
        for (r0, r1, Pp, (c0, c1, Qp)) in parts:
            Pg[r0:r1] = Pp
            Qg[c0:c1] = Qp
        np.save(out + "_P.npy", Pg)
        np.save(out + "_Q.npy", Qg)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("G,Br,Bc,sched,sync", [
    (2, 3, 6, "det", "ring"), (3, 2, 6, "det", "ring"), (2, 1, 4, "hogwild", "ring"),
    (2, 3, 3, "det", "allreduce"), (3, 1, 1, "hogwild", "allreduce"),
])
def test_distributed_schedule_matches_oracle(tmp_path, G, Br, Bc, sched, sync):
    import __graft_entry__
    __graft_entry__.build()
    out = str(tmp_path / "res")
    epochs = 2
    mp.spawn(_worker, args=(G, Br, Bc, sched, sync, epochs, _free_port(), out), nprocs=G, join=True)
    Pg, Qg = np.load(out + "_P.npy"), np.load(out + "_Q.npy")
    ref = _problem(G, Br, Bc)
    osched = "det" if sched == "det" else "serial"
    for _ in range(epochs):
        ref.epoch(osched, sync)
    assert not np.isnan(Pg).any() and not np.isnan(Qg).any()
    if sync == "ring":  # serialisable: bit-exact
        assert np.array_equal(Pg, ref.P) and np.array_equal(Qg, ref.Q)
    else:  # the mean is summed in another order
        np.testing.assert_allclose(Pg, ref.P, rtol=0, atol=1e-12)
        np.testing.assert_allclose(Qg, ref.Q, rtol=0, atol=1e-12)
