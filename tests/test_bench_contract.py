"""bench.py's roofline arithmetic on CPU (no device): the JSON line's `roofline` object follows the
recipe of DESIGN.md section 8 -- achieved = ALGORITHMIC bytes per launch (every local
record once + the rank's P rows and Q read and written once) / the launch's duration, frac =
achieved / peak (an HBM fraction, <= 1 for any real launch), north_star_frac with the north_star's
12 + 16k bytes per update, binding_frac = the in-run ceiling probe's time / the kernel's time, and
the DET latency roof; traffic comes from the committed ncu capture table."""
import importlib.util
import os

import pytest

import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod


def test_c5_algorithmic_bytes_and_fractions(bench):
    cfg = synth.CONFIGS["c5"]
    info = {"local_nnz": cfg.nnz, "rows": cfg.m}
    r = bench.roofline(cfg, "c5", "fp32", "hogwild", info, kmean_ms=320.0, step_ms=321.0, peak=6551.0,
                       peak_src="test", probe=("red_f32", 260.0, 330.0))
    alg = 12 * cfg.nnz + 2 * cfg.m * cfg.k * 4 + 2 * cfg.n * cfg.k * 4
    assert r["algorithmic_bytes_per_launch"] == alg
    assert r["algorithmic_bytes_per_update"] == pytest.approx(28.556, abs=1e-3)  # C5 28.6 B
    assert r["achieved"] == pytest.approx(alg / 0.320 / 1e9)
    assert r["frac"] == pytest.approx(r["achieved"] / 6551.0) and r["frac"] < 1.0
    assert r["north_star_bytes_per_update"] == 12 + 16 * cfg.k == 2060
    assert r["north_star_frac"] == pytest.approx(cfg.nnz * 2060 / 0.320 / 1e9 / 6551.0)
    assert r["binding_frac"] == pytest.approx(260.0 / 320.0)
    assert r["roundtrip_frac"] == pytest.approx(330.0 / 320.0)
    assert r["bound"] == "l2_atomic" and r["kernel_share_of_step"] == pytest.approx(320.0 / 321.0)
    assert r["traffic"] == bench.ncu_traffic("c5/hogwild") and r["traffic_key"] == "c5/hogwild"


def test_binary16_storage_bytes(bench):
    cfg = synth.CONFIGS["c3"]
    info = {"local_nnz": cfg.nnz, "rows": cfg.m}
    r = bench.roofline(cfg, "c3", "fp16sr", "hogwild", info, 8.0, 8.1, 6551.0, "test", ("ldred_f16", 8.0))
    assert r["algorithmic_bytes_per_launch"] == 12 * cfg.nnz + 2 * cfg.m * cfg.k * 4 + 2 * cfg.n * cfg.k * 2
    assert r["north_star_bytes_per_update"] == 12 + 12 * cfg.k
    assert r["traffic_key"] == "c3-fp16sr/hogwild" and "roundtrip_frac" not in r


def test_det_latency_roof(bench):
    cfg = synth.CONFIGS["c3"]
    info = {"local_nnz": cfg.nnz, "rows": cfg.m}
    probe = {"critical_ratings": 135000, "chain_ns_per_rating": 160.0, "ms": 135000 * 160.0 / 1e6}
    r = bench.roofline(cfg, "c3", "fp32", "det", info, 29.0, 29.2, 6551.0, "test", probe)
    assert r["bound"] == "latency" and r["traffic_key"] == "c3/det"
    assert r["binding_frac"] == pytest.approx(21.6 / 29.0)
    assert r["binding_ceiling"] is probe
