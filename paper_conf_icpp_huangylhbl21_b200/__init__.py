"""B200-native hot path of HCC-MF (Huang et al., ICPP '21): thin Python binding.

Argument marshalling only.  Every step of the path (ingest, shuffle, partition,
sort, SGD epoch, Q synchronisation, RMSE, export) runs in libhccmf.so's CUDA
kernels behind the C ABI declared in include/hccmf.h; torch is used only for
device memory, streams and the process group that bootstraps NCCL.  There is
no CPU fallback: if libhccmf.so is missing the import of this module fails.

    model = Model(m, n, k, gamma=0.005, lam=0.01)
    model.load(u, v, r)                      # int32 / int32 / float32, numpy or torch (CPU or CUDA)
    model.partition(n_shards=1, grid=(1, 1), strategy="DP0", seed=1)
    model.init(seed=7)                       # or model.set_factors(P0, Q0)
    for _ in range(epochs):
        model.train_epoch("hogwild", sync="none")
    rmse = model.rmse(tu, tv, tr)
    P, Q = model.factors()

Multi-rank: ``Model(..., dist=True)`` under torchrun (NCCL, one process per GPU), or
``Model(..., hub=Hub(G), rank=r)`` from G host threads of one process: the loopback
data plane on one device (same call sites and buffers as NCCL; tests).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("HCCMF_LIB") or os.path.join(_HERE, "libhccmf.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback)")

OK, EINVAL, ERANGE, ENOMEM, ESTATE, ECUDA, ENCCL = 0, -1, -2, -3, -4, -5, -6
STATUS = {0: "OK", -1: "EINVAL", -2: "ERANGE", -3: "ENOMEM", -4: "ESTATE", -5: "ECUDA", -6: "ENCCL"}
SCHED = {"det": 0, "hogwild": 1}
SYNC = {"none": 0, "ring": 1, "allreduce": 2}
DP = {"DP0": 0, "DP1": 1, "DP2": 2}
OPT = {"hogwild_warps": 1, "task_ratings": 2, "sync_stream": 3, "hogwild_atomic": 5, "conflict_ratio": 6, "heavy_first": 7, "vec": 8, "det_wave": 9, "sync_phases": 10, "wire_fp16": 11, "l2_persist": 12, "prefetch_depth": 13, "storage": 14, "timeline": 15, "staleness": 16}


class HccmfError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"hccmf {STATUS.get(code, code)}: {msg}")
        self.code = code


class PartitionOpts(ctypes.Structure):
    _fields_ = [("n_shards", ctypes.c_int32), ("grid_rows", ctypes.c_int32), ("grid_cols", ctypes.c_int32),
                ("strategy", ctypes.c_int32), ("x", ctypes.c_void_p), ("t_meas", ctypes.c_void_p),
                ("t_sync", ctypes.c_double), ("seed", ctypes.c_uint64), ("storage", ctypes.c_int32),
                ("grid_dim", ctypes.c_int32), ("col_balance", ctypes.c_int32)]


class Info(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("k", ctypes.c_int32),
                ("n_shards", ctypes.c_int32), ("shard_lo", ctypes.c_int32), ("shard_hi", ctypes.c_int32),
                ("local_nnz", ctypes.c_int64), ("row0", ctypes.c_int64), ("rows", ctypes.c_int64),
                ("n_blocks", ctypes.c_int64), ("n_tasks", ctypes.c_int64), ("key_bits", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("device_bytes", ctypes.c_int64),
                ("transposed", ctypes.c_int32), ("det_path", ctypes.c_int32)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = None


def lib():
    """Load libhccmf.so and declare the C ABI (include/hccmf.h)."""
    global _lib
    if _lib is None:
        L = ctypes.CDLL(LIB_PATH)
        P, i32, i64, u64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_float
        st = ctypes.c_int
        sig = {
            "hccmf_create": (st, [i64, i64, i32, f32, f32, P]),
            "hccmf_nccl_unique_id": (st, [P]),
            "hccmf_create_dist": (st, [i64, i64, i32, f32, f32, P, i32, i32, i32, P]),
            "hccmf_set_stream": (st, [P, P]),
            "hccmf_set_option": (st, [P, i32, i64]),
            "hccmf_destroy": (None, [P]),
            "hccmf_last_error": (ctypes.c_char_p, [P]),
            "hccmf_load_ratings": (st, [P, P, P, P, i64]),
            "hccmf_partition": (st, [P, ctypes.POINTER(PartitionOpts)]),
            "hccmf_init_factors": (st, [P, u64]),
            "hccmf_set_factors": (st, [P, P, P]),
            "hccmf_train_epoch": (st, [P, i32, i32]),
            "hccmf_rmse": (st, [P, P, P, P, i64, ctypes.POINTER(ctypes.c_double)]),
            "hccmf_get_factors": (st, [P, P, P]),
            "hccmf_get_partition": (st, [P, P, P, P, P]),
            "hccmf_get_records": (st, [P, P, P, P]),
            "hccmf_get_fractions": (st, [P, P]),
            "hccmf_get_info": (st, [P, ctypes.POINTER(Info)]),
            "hccmf_version": (ctypes.c_char_p, []),
            "hccmf_hub_create": (st, [i32, P]),
            "hccmf_hub_destroy": (None, [P]),
            "hccmf_create_loopback": (st, [i64, i64, i32, f32, f32, P, i32, i32, P]),
            "hccmf_comm_counts": (st, [P, P, i32, P]),
            "hccmf_load_ratings_slice": (st, [P, P, P, P, i64]),
            "hccmf_probe_roundtrip": (st, [P, i32, i64, i32, ctypes.POINTER(ctypes.c_double)]),
            "hccmf_timeline": (st, [P, P, i64, P]),
            "hccmf_kernel_launches": (ctypes.c_int64, []),
            "hccmf_schedule": (st, [i32, i32, i32, i64, i32, i32, i32, P, P, P, P, P, P]),
            "hccmf_cost_model": (st, [i32, i64, i64, i64, i32, P, P, ctypes.c_double, i32, i32, i32,
                                      ctypes.c_double, P, P, P, P, P]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def kernel_launches() -> int:
    """Kernels the library has launched in this process (hccmf_kernel_launches)."""
    return int(lib().hccmf_kernel_launches())


def version() -> str:
    return lib().hccmf_version().decode()


def _buf(x, dtype):
    """(pointer, keepalive) for a numpy array or torch tensor of the given numpy dtype."""
    if x is None:
        return None, None
    try:
        import torch
        if isinstance(x, torch.Tensor):
            tdt = {np.int32: torch.int32, np.float32: torch.float32, np.float64: torch.float64,
                   np.int64: torch.int64}[np.dtype(dtype).type]
            t = x.contiguous().to(tdt)
            return t.data_ptr(), t
    except ImportError:  # pragma: no cover
        pass
    a = np.ascontiguousarray(x, dtype=dtype)
    return a.ctypes.data, a


def schedule(G, Br, Bc, n, sched="det", sync="none", shard=-1):
    """The launch/block schedule (and ring exchange ranges) one shard executes; host-only."""
    L = lib()
    nb, nl = ctypes.c_int64(0), ctypes.c_int64(0)
    code = L.hccmf_schedule(G, Br, Bc, n, SCHED[sched], SYNC[sync], shard, None, ctypes.byref(nb), None, None,
                            ctypes.byref(nl), None)
    if code != OK:
        raise HccmfError(code, L.hccmf_last_error(None).decode())
    blocks = np.empty(nb.value, np.int64)
    off = np.empty(nl.value + 1, np.int64)
    stage = np.empty(nl.value, np.int32)
    ring = np.zeros((G, 4), np.int64)
    code = L.hccmf_schedule(G, Br, Bc, n, SCHED[sched], SYNC[sync], shard, blocks.ctypes.data, ctypes.byref(nb),
                            off.ctypes.data, stage.ctypes.data, ctypes.byref(nl), ring.ctypes.data)
    if code != OK:
        raise HccmfError(code, L.hccmf_last_error(None).decode())
    launches = [blocks[off[i]:off[i + 1]] for i in range(nl.value)]
    return launches, stage, ring


def cost_model(m, n, nnz, k, B, Bbus, B_server, t=1, q_only=True, elem_bytes=4, lambda_sync=10.0):
    """Section 3.2 time cost model (Eq. 1-5): returns (x, T_i, T_sync, T, strategy name)."""
    B = np.ascontiguousarray(B, np.float64)
    Bbus = np.ascontiguousarray(Bbus, np.float64)
    p = len(B)
    x, Ti = np.empty(p), np.empty(p)
    Ts, T, strat = ctypes.c_double(), ctypes.c_double(), ctypes.c_int32()
    L = lib()
    code = L.hccmf_cost_model(p, m, n, nnz, k, B.ctypes.data, Bbus.ctypes.data, float(B_server), t, int(q_only),
                              elem_bytes, float(lambda_sync), x.ctypes.data, Ti.ctypes.data, ctypes.byref(Ts),
                              ctypes.byref(T), ctypes.byref(strat))
    if code != OK:
        raise HccmfError(code, L.hccmf_last_error(None).decode())
    return x, Ti, Ts.value, T.value, {1: "DP1", 2: "DP2"}[strat.value]


COMM_SITES = ("ring_stage", "ring_block", "ring_wire16", "materialize_q", "allreduce_q", "allreduce_q16",
              "rmse", "export_p", "ingest_hist", "ingest_exchange", "ingest_blocks")


class Hub:
    """Loopback communicator hub for `world` ranks of this process (hccmf_hub_create)."""

    def __init__(self, world):
        self.world = int(world)
        self._p = ctypes.c_void_p()
        code = lib().hccmf_hub_create(self.world, ctypes.byref(self._p))
        if code != OK:
            raise HccmfError(code, "hccmf_hub_create")

    def close(self):
        if getattr(self, "_p", None):
            lib().hccmf_hub_destroy(self._p)
            self._p = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # pragma: no cover
            pass


class Model:
    """One handle of libhccmf (single process, or one rank of a distributed job)."""

    def __init__(self, m, n, k, gamma=0.005, lam=0.01, *, dist=False, device=None, hub=None, rank=None):
        self.m, self.n, self.k, self.gamma, self.lam = int(m), int(n), int(k), float(gamma), float(lam)
        self._h = ctypes.c_void_p()
        L = lib()
        if hub is not None:
            dev = 0 if device is None else int(device)
            self._check(L.hccmf_create_loopback(self.m, self.n, self.k, self.gamma, self.lam, hub._p, int(rank), dev,
                                                ctypes.byref(self._h)))
        elif dist:
            import torch
            import torch.distributed as tdist
            rank, world = tdist.get_rank(), tdist.get_world_size()
            if device is None:
                device = int(os.environ.get("LOCAL_RANK", rank % max(1, torch.cuda.device_count())))
            uid = (ctypes.c_uint8 * 128)()
            if rank == 0:
                self._check(L.hccmf_nccl_unique_id(uid))
            t = torch.tensor(list(bytes(uid)), dtype=torch.uint8)
            if tdist.get_backend() == "nccl":
                t = t.cuda(device)
            tdist.broadcast(t, 0)
            uid = (ctypes.c_uint8 * 128)(*t.cpu().tolist())
            self._check(L.hccmf_create_dist(self.m, self.n, self.k, self.gamma, self.lam, uid, rank, world, device,
                                            ctypes.byref(self._h)))
        else:
            if device is not None:
                import torch
                torch.cuda.set_device(device)
            self._check(L.hccmf_create(self.m, self.n, self.k, self.gamma, self.lam, ctypes.byref(self._h)))
        self.G = 1

    # -------------------------------------------------------------- plumbing
    def _check(self, code):
        if code != OK:
            msg = lib().hccmf_last_error(self._h if getattr(self, "_h", None) else None)
            raise HccmfError(code, msg.decode() if msg else "")

    def close(self):
        if getattr(self, "_h", None):
            lib().hccmf_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # pragma: no cover
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def set_stream(self, stream):
        """Issue all work on a torch.cuda.Stream (or raw cudaStream_t int)."""
        handle = getattr(stream, "cuda_stream", stream)
        self._check(lib().hccmf_set_stream(self._h, ctypes.c_void_p(int(handle))))

    def set_option(self, name, value):
        self._check(lib().hccmf_set_option(self._h, OPT[name], int(value)))

    # ------------------------------------------------------------- the path
    def load(self, u, v, r):
        pu, ku = _buf(u, np.int32)
        pv, kv = _buf(v, np.int32)
        pr, kr = _buf(r, np.float32)
        nnz = len(ku)
        assert len(kv) == nnz and len(kr) == nnz, "u, v, r must have the same length"
        self._check(lib().hccmf_load_ratings(self._h, pu, pv, pr, nnz))

    def load_slice(self, u, v, r):
        """This rank's slice of the global COO (hccmf_load_ratings_slice): ranks' slices in
        rank order concatenate to the global COO; partition then shards without copies."""
        pu, ku = _buf(u, np.int32)
        pv, kv = _buf(v, np.int32)
        pr, kr = _buf(r, np.float32)
        nnz = len(ku)
        assert len(kv) == nnz and len(kr) == nnz, "u, v, r must have the same length"
        self._check(lib().hccmf_load_ratings_slice(self._h, pu, pv, pr, nnz))

    def probe_roundtrip(self, mode="red_f32", warps=0, reps=3) -> float:
        """Mean ms of one pass of the q_v round-trip ceiling probe (hccmf_probe_roundtrip)."""
        out = ctypes.c_double()
        m = {"red_f32": 0, "ldred_f16": 1, "ldred_f32": 2, "q_stream": 3, "p_stream": 4, "bulkred_f32": 5, "bulkldred_f32": 6,
             "ldbulkred_f32": 7, "bulkldred8_f32": 8, "bulkldred2_f32": 9}[mode]
        self._check(lib().hccmf_probe_roundtrip(self._h, m, int(warps), int(reps), ctypes.byref(out)))
        return out.value

    def timeline(self):
        """Rows {kind, stage, block, start ms, end ms} of the last epoch (HCCMF_OPT_TIMELINE)."""
        n = ctypes.c_int64()
        self._check(lib().hccmf_timeline(self._h, None, 0, ctypes.byref(n)))
        rows = np.zeros((n.value, 5), np.float64)
        if n.value:
            self._check(lib().hccmf_timeline(self._h, rows.ctypes.data, n.value, ctypes.byref(n)))
        return rows

    def comm_counts(self) -> dict:
        """How many times each data-plane call site ran on this handle (hccmf_comm_counts)."""
        c = np.zeros(len(COMM_SITES), np.int64)
        ns = ctypes.c_int32()
        self._check(lib().hccmf_comm_counts(self._h, c.ctypes.data, len(c), ctypes.byref(ns)))
        assert ns.value == len(COMM_SITES)
        return dict(zip(COMM_SITES, c.tolist()))

    def partition(self, n_shards=1, grid=(1, 1), strategy="DP0", seed=0, x=None, t_meas=None, t_sync=0.0,
                  grid_dim="rows", storage="fp32", col_balance=False):
        """grid_dim: "rows" (shards of users, Q moves), "cols" (shards of items, P moves) or
        "auto" (the paper's rule, L884-L886).  storage: "fp32"; "fp16" = Q held in IEEE
        binary16 during epochs, fp32 arithmetic, round to nearest (R26; k a multiple
        of 128); "fp16sr" = the same with stochastic rounding of every q write (R27).
        col_balance: degree-balanced column blocks instead of the hash shuffle of columns (R30)."""
        px, kx = _buf(x, np.float64)
        pt, kt = _buf(t_meas, np.float64)
        o = PartitionOpts(int(n_shards), int(grid[0]), int(grid[1]), DP[strategy] if isinstance(strategy, str)
                          else int(strategy), px, pt, float(t_sync), int(seed), {"fp32": 0, "fp16": 1, "fp16sr": 2}[storage],
                          {"rows": 0, "cols": 1, "auto": 2}[grid_dim], int(bool(col_balance)))
        self._check(lib().hccmf_partition(self._h, ctypes.byref(o)))
        self.G, self.grid = int(n_shards), (int(grid[0]), int(grid[1]))

    def init(self, seed):
        self._check(lib().hccmf_init_factors(self._h, int(seed)))

    def set_factors(self, P, Q):
        pP, kP = _buf(P, np.float32)
        pQ, kQ = _buf(Q, np.float32)
        assert kP.shape == (self.m, self.k) and kQ.shape == (self.n, self.k)
        self._check(lib().hccmf_set_factors(self._h, pP, pQ))

    def train_epoch(self, sched="hogwild", sync="none"):
        self._check(lib().hccmf_train_epoch(self._h, SCHED[sched], SYNC[sync]))

    def rmse(self, u, v, r) -> float:
        pu, ku = _buf(u, np.int32)
        pv, kv = _buf(v, np.int32)
        pr, kr = _buf(r, np.float32)
        out = ctypes.c_double()
        self._check(lib().hccmf_rmse(self._h, pu, pv, pr, len(ku), ctypes.byref(out)))
        return out.value

    def factors(self, P=None, Q=None, want_P=True, want_Q=True):
        """P (m x k), Q (n x k) in original id order.  Host numpy by default; pass
        preallocated torch CUDA tensors to receive them on the device."""
        if want_P and P is None:
            P = np.empty((self.m, self.k), np.float32)
        if want_Q and Q is None:
            Q = np.empty((self.n, self.k), np.float32)
        pP = (P.data_ptr() if hasattr(P, "data_ptr") else P.ctypes.data) if want_P else None
        pQ = (Q.data_ptr() if hasattr(Q, "data_ptr") else Q.ctypes.data) if want_Q else None
        self._check(lib().hccmf_get_factors(self._h, pP, pQ))
        return P, Q

    # --------------------------------------------------------- introspection
    def info(self) -> dict:
        i = Info()
        self._check(lib().hccmf_get_info(self._h, ctypes.byref(i)))
        return i.as_dict()

    def get_partition(self):
        inf = self.info()
        b = np.empty(inf["n_shards"] + 1, np.int32)
        off = np.empty(inf["n_blocks"] + 1, np.int64)
        pr = np.empty(inf["m"], np.int32)
        pc = np.empty(inf["n"], np.int32)
        self._check(lib().hccmf_get_partition(self._h, b.ctypes.data, off.ctypes.data, pr.ctypes.data,
                                              pc.ctypes.data))
        return b, off, pr, pc

    def records(self):
        c = self.info()["local_nnz"]
        u = np.empty(c, np.int32)
        v = np.empty(c, np.int32)
        r = np.empty(c, np.float32)
        self._check(lib().hccmf_get_records(self._h, u.ctypes.data, v.ctypes.data, r.ctypes.data))
        return u, v, r

    def fractions(self):
        x = np.empty(self.G, np.float64)
        self._check(lib().hccmf_get_fractions(self._h, x.ctypes.data))
        return x
