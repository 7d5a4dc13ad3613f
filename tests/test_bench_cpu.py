"""bench.py's host-side arithmetic (no GPU): the per-pass binding bound, the shared config of
both arms, and the workload table (BASELINE.json configs)."""
import importlib.util
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_per_pass_binding(bench):
    """bound = max(bytes / HBM peak, FP64 / FP64 peak) per pass; frac = sum bound / sum measured."""
    prof = [
        {"kind": 0, "k_in": 30, "k_out": 30, "n_gates": 10, "ms": 10.0, "bytes": 65e9,
         "amps_computed": 2 ** 30, "fp64_ops": 0.0, "lane_ops": 0, "remaps": 0},          # HBM: 10 ms
        {"kind": 0, "k_in": 30, "k_out": 30, "n_gates": 40, "ms": 40.0, "bytes": 6.5e9,
         "amps_computed": 2 ** 30, "fp64_ops": 16e12 * 0.02, "lane_ops": 2, "remaps": 1},  # FP64: 20 ms
    ]
    b = bench.per_pass_binding(prof, 6500.0, 16e12)
    assert b["passes"][0]["binding"] == "hbm" and abs(b["passes"][0]["hbm_ms"] - 10.0) < 1e-9
    assert b["passes"][1]["binding"] == "fp64" and abs(b["passes"][1]["fp64_ms"] - 20.0) < 1e-9
    assert abs(b["bound_ms"] - 30.0) < 1e-9 and abs(b["measured_ms"] - 50.0) < 1e-9
    assert abs(b["frac"] - 0.6) < 1e-12
    # the supplementary SM-side bound adds the MIO time of lane ops / remaps to the FP64 time
    assert b["sm_bound"]["bound_ms"] > b["bound_ms"]
    assert b["passes"][1]["mio_ms"] > 0 and b["passes"][0]["mio_ms"] == 0


def test_reference_and_gpu_arm_share_the_config(bench):
    import argparse
    args = argparse.Namespace(reorder=2, no_prune=False, fuse_bits=12)
    circ, desc = bench.workload("qaoa32", None)
    a = bench.run_config(args, circ, desc, 1)
    b = bench.run_config(args, circ, desc, 1)
    assert a == b and a["n_qubits"] == 32 and a["gates"] == 384
    assert "configs[2]" in desc


def test_workloads_match_baseline_configs(bench):
    """configs[1]: QFT_28 (420 gates: 28 H + 378 CP + 14 SWAP); |x> adds the X gates of x."""
    c, _ = bench.workload("qft28", None)
    assert c.n == 28 and len(c.ops) == 420
    cx, _ = bench.workload("qft28x", None)
    x = bench.qft_x(28)
    assert len(cx.ops) == 420 + bin(x).count("1") and 0 <= x < 2 ** 28
    r, _ = bench.workload("rqc", 34)
    assert r.n == 34
