"""CPU-only checks of the C ABI library: it builds/loads, exports every declared symbol, and its
host logic (QASM loader, Alg.2/3 reorder, pass planner) agrees with the oracle. No GPU calls."""
import os
import re

import numpy as np
import pytest

from oracle import qasm as oq
from oracle import schedule as osch
from workloads import circuits as wc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def q():
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


def test_exports_every_declared_symbol(q):
    hdr = open(os.path.join(ROOT, "include", "qgpu.h")).read()
    declared = set(re.findall(r"\b(qgpu_[a-z_]+)\s*\(", hdr))
    assert len(declared) >= 20
    lib = q.load()
    for name in declared:
        assert hasattr(lib, name), name
    assert declared <= set(q.EXPORTS) | {"qgpu_last_error", "qgpu_version"}
    assert "sm_100a" in q.version()


def test_config_struct_size(q):
    import ctypes
    cfg = q.config()
    assert cfg.struct_size == ctypes.sizeof(q.Config)
    assert (cfg.prune, cfg.reorder, cfg.chunk_bits, cfg.fuse_bits, cfg.world_size) == (1, 2, 21, 12, 1)


CIRCS = {
    "ghz_qft5": lambda: wc.ghz_qft(5),
    "qft12": lambda: wc.qft(12),
    "qft9x": lambda: wc.qft(9, x=300),
    "qaoa14": lambda: wc.qaoa(14, 2, seed=1),
    "rqc12": lambda: wc.rqc(12, 10, seed=3),
    "gs3x4": lambda: wc.gs(3, 4),
    "hlf3x4": lambda: wc.hlf(3, 4, seed=2),
    "bv9": lambda: wc.bv(9, 0b10110101),
    "iqp8": lambda: wc.iqp(8),
    "rand8": lambda: wc.random_circuit(8, 150, seed=11),
    "rand10": lambda: wc.random_circuit(10, 300, seed=12),
}


@pytest.mark.parametrize("name", sorted(CIRCS))
def test_loader_matches_oracle_parser(q, name):
    c = CIRCS[name]()
    text = c.qasm()
    n, gates = oq.parse(text)
    qc = q.Circuit(text)
    assert qc.info() == (n, len(gates))


@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("mode", [0, 1, 2])
def test_reorder_bit_exact_vs_oracle(q, name, mode):
    """oracle and library schedules must be identical (Alg.2/Alg.3 + Q4)."""
    c = CIRCS[name]()
    text = c.qasm()
    _, gates = oq.parse(text)
    ref = osch.reorder(gates, mode)
    got = q.Circuit(text).reorder(mode)
    assert list(got) == list(ref)


@pytest.mark.parametrize("name", sorted(CIRCS) + ["randdiag"])
@pytest.mark.parametrize("mode", [0, 1, 2])
def test_reorder_refined_rule_bit_exact_vs_oracle(q, name, mode):
    """NEXT-1: with the refined involvement rule (mode + 4) the Alg.2/Alg.3 costs count only the
    qubits a gate would involve; library and oracle schedules stay identical."""
    c = CIRCS[name]() if name in CIRCS else wc.random_circuit(
        9, 120, seed=13, names=["cp", "cz", "rz", "cx", "crx", "ccx", "t", "h", "rzz", "cswap", "x"])
    text = c.qasm()
    _, gates = oq.parse(text)
    ref = osch.reorder(gates, mode, rule=1)
    got = q.Circuit(text).reorder(mode + 4)
    assert list(got) == list(ref)
    assert osch.is_topological(gates, list(got))


def test_reorder_gs5_walkthrough(q):
    """forward-looking reorder of the gs_5 example gives 1,2,2,3,3,4,4,4,5."""
    text = ('OPENQASM 2.0;\ninclude "qelib1.inc";\nqreg q[5];\nh q[0];\nh q[1];\nh q[2];\nh q[3];\n'
            'h q[4];\ncx q[0],q[1];\ncx q[0],q[2];\ncx q[1],q[3];\ncx q[2],q[3];\n')
    order = q.Circuit(text).reorder(2)
    _, gates = oq.parse(text)
    cnt = [bin(i).count("1") for i in osch.involvement_trace(gates, list(order))]
    assert cnt == [1, 2, 2, 3, 3, 4, 4, 4, 5]


@pytest.mark.parametrize("name", ["qft12", "qaoa14", "rqc12", "rand10", "hlf3x4"])
@pytest.mark.parametrize("fuse", [0, 7, 9, 12])
def test_plan_invariants(q, name, fuse):
    """a4: passes are consecutive runs of the reordered list; tile passes have <= b tile bits
    that include the low contiguous run; live sizes never shrink."""
    c = CIRCS[name]()
    qc = q.Circuit(c.qasm())
    n, ng = qc.info()
    plan = qc.plan(n, 1, 2, fuse)
    pos = 0
    k_prev = 0
    for first, count, kind, kin, kout, b, slo, shi in plan:
        assert first == pos and (count >= 1 or kind == 7)  # 7: zero-half materialisation
        pos += count
        assert kin == k_prev and kout >= kin
        k_prev = kout
        if kind == 7:
            continue
        if fuse == 0:
            assert kind in (1, 2, 3, 4)
            assert count >= 1  # > 1 when CX.D.CX triples are fused into one diagonal gate
        else:
            assert kind in (0, 4)
            if kind == 0:
                S = int(slo) | (int(shi) << 32)
                assert bin(S).count("1") == b <= fuse
                assert b == min(fuse, kout)
                # the lane-bit policies the planner may pick (plan_circuit_auto) keep
                # at least the 3 lowest positions (128-byte runs per warp access) in every tile
                lm = min(3, kout)
                assert S & ((1 << lm) - 1) == (1 << lm) - 1
                assert S >> kout == 0
    assert pos == ng
    assert k_prev == n or ng == 0 or k_prev == bin(osch.involvement_trace(oq.parse(c.qasm())[1])[-1]).count("1")


@pytest.mark.parametrize("name", ["qft12", "qft9x", "rand10", "hlf3x4", "ghz_qft5"])
@pytest.mark.parametrize("fuse", [0, 9, 12])
def test_plan_invariants_refined_rule(q, name, fuse):
    """NEXT-1 plans (reorder + 4): still consecutive runs covering every gate (skipped gates are
    counted in the pass they fall in), live sizes never shrink, and the final live size is the
    refined involvement of the oracle replay."""
    c = CIRCS[name]()
    text = c.qasm()
    qc = q.Circuit(text)
    n, ng = qc.info()
    _, gates = oq.parse(text)
    plan = qc.plan(n, 1, 6, fuse)
    pos, k_prev = 0, 0
    for first, count, kind, kin, kout, b, slo, shi in plan:
        assert first == pos and (count >= 1 or kind == 7)
        pos += count
        assert kin == k_prev and kout >= kin
        k_prev = kout
    assert pos == ng
    inv = osch.involvement_trace(gates, osch.reorder(gates, 2, rule=1), rule=1)[-1]
    assert k_prev == bin(inv).count("1")


def test_pass_schedule_cuts_qaoa32_traffic(q, monkeypatch):
    """Pass-aware execution order (DESIGN.md §4 "Pass scheduling"): QAOA_32 (configs[2]) planned
    over the commutation DAG moves well under half the bytes of the consecutive-run plan (round 2:
    499 GB -> 157 GB per circuit, no pass at the full live size before the last involvement); the
    plan stays a sequence of consecutive runs covering every gate with non-shrinking live sizes."""
    c = wc.qaoa(32, 2, seed=1)

    def plan(sched):
        monkeypatch.setenv("QGPU_PASS_SCHED", sched)
        return q.Circuit(c.qasm()).plan(32, 1, 2, 12)

    def traffic(p):
        return sum(2.0 ** r[3] + 2.0 ** r[4] for r in p if r[2] == 0) * 16

    old, new = plan("0"), plan("1")
    assert traffic(new) < 0.4 * traffic(old)
    assert sum(1 for r in new if r[3] == 32) == 0  # every pass still expands
    pos, k_prev = 0, 0
    for first, count, kind, kin, kout, *_ in new:
        assert first == pos and count >= 1 and kind == 0 and kin == k_prev and kout >= kin
        pos += count
        k_prev = kout
    assert pos == q.Circuit(c.qasm()).info()[1] and k_prev == 32


def test_fused_qft28_is_few_passes(q):
    """QFT_28 (config C2) with Alg.3 and b=12 collapses into a handful of HBM passes."""
    qc = q.Circuit(wc.qft(28).qasm())
    plan = qc.plan(28, 1, 2, 12)
    assert len(plan) <= 40


def test_parse_errors(q):
    with pytest.raises(q.QgpuError) as e:
        q.Circuit("OPENQASM 2.0;\nqreg q[2];\nh q[0]\ncx q[0],q[1];\n")
    assert e.value.kind == "PARSE" and "line 4" in str(e.value)
    with pytest.raises(q.QgpuError) as e:
        q.Circuit("OPENQASM 2.0;\nqreg q[2];\nreset q[0];\n")
    assert e.value.kind == "UNSUPPORTED"
    with pytest.raises(q.QgpuError) as e:
        q.Circuit("OPENQASM 2.0;\nqreg q[2];\nfoo q[0];\n")
    assert e.value.kind == "UNSUPPORTED"
    with pytest.raises(q.QgpuError) as e:
        q.Circuit("OPENQASM 2.0;\nqreg q[2];\ncx q[0],q[0];\n")
    assert e.value.kind == "INVALID_ARG"
    # statements that repeat a gate name (the parser reuses the matrix of an identical name +
    # parameter text) still get every check of their own
    for text, kind in (("h q[0];\nh(", "PARSE"), ("rx(0.1) q[0];\nrx(0.1 q[0];", "PARSE"),
                       ("rx(0.1) q[0];\nrx(0.1) q[0],q[1];", "INVALID_ARG"),
                       ("h q[0];\nh(0.1) q[0];", "INVALID_ARG"), ("cx q[0],q[1];\ncx q[1],q[1];", "INVALID_ARG")):
        with pytest.raises(q.QgpuError) as e:
            q.Circuit("OPENQASM 2.0;\nqreg q[2];\n" + text + "\n")
        assert e.value.kind == kind, text
    c = q.Circuit("OPENQASM 2.0;\nqreg a[2];\nqreg b[3];\ncreg c[5];\nh b;\ncx a[1],b[2];\n"
                  "rx(-pi/2^2 + 2*sin(pi/6)) a[0];\nbarrier a;\nmeasure a[0] -> c[0];\n")
    assert c.info() == (5, 5)


def test_state_create_without_gpu_fails_cleanly(q):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(q.QgpuError) as e:
        q.State(10)
    assert e.value.kind in ("CUDA", "OUT_OF_MEMORY")


def test_jit_sources_compile_without_gpu(q):
    """The per-pass NVRTC sources compile for sm_100a on the CPU box (no GPU)."""
    for c in (wc.ghz_qft(5), wc.random_circuit(9, 80, seed=3)):
        qc = q.Circuit(c.qasm())
        try:
            k = qc.jit_check(c.n, 2, 7)
        except q.QgpuError as e:
            if e.kind == "UNSUPPORTED":
                pytest.skip("NVRTC not available")
            raise
        n_tile = sum(1 for r in qc.plan(c.n, 1, 2, 7) if r[2] == 0)
        assert k == n_tile


def test_jit_sources_specialise_the_fp64_bound_passes(q, monkeypatch, tmp_path):
    """Round-2 NVRTC specialisations, checked in the generated sources of QAOA_16 (whose plan has
    the same structure as QAOA_32's) and compiled for sm_100a on the CPU box: the tile-uniform
    scalar joins the first phase run (kScalarFolded), programs with <= 2 remaps hand the buffer
    to the next tile's loads after their last remap (pf()), and the fused-measurement variants
    -- modes 0/1/2 and mode 2 with compile-time reduce-scatter masks and global reductions
    (QGPU_JIT_CHECK_HIST key 0x131f: lane bits 0-4 unrequested, register bits 0-1 dead) --
    compile."""
    c = wc.qaoa(16, 2, seed=1)
    monkeypatch.setenv("QGPU_JIT_DUMP", str(tmp_path))
    monkeypatch.setenv("QGPU_JIT_CACHE", str(tmp_path / "cache"))
    monkeypatch.setenv("QGPU_JIT_CHECK_HIST", "0x131f")
    qc = q.Circuit(c.qasm())
    try:
        k = qc.jit_check(c.n, 2, 12)
    except q.QgpuError as e:
        if e.kind == "UNSUPPORTED":
            pytest.skip("NVRTC not available")
        raise
    n_tile = sum(1 for r in qc.plan(c.n, 1, 2, 12) if r[2] == 0)
    assert k == n_tile + 4
    srcs = [p.read_text() for p in tmp_path.glob("qgpu_pass_*.cu")]
    plain = [t for t in srcs if "kHist = false" in t]
    assert len(plain) == n_tile
    assert any("kScalarFolded = true" in t for t in plain)
    for t in plain:  # the scalar is folded exactly when the program has a phase run
        if "kHasScalar = true" in t:
            assert ("kScalarFolded = true" in t) == ("run_apply_" in t)
        assert t.count("pf();") <= 1
        if "pf();" in t:
            assert "kEarlyPrefetch = true" in t and t.count("tile_reload_j") <= 2 + 1
    rs = [t for t in srcs if "kHistRS = true" in t]
    assert len(rs) == 1 and "kHlred = 31u" in rs[0] and "kDead = 3u" in rs[0] and "kHistGlob = true" in rs[0]


def test_fusion_lookahead_cuts_hbm_passes(q, monkeypatch):
    """Fusion lookahead (planner): commuting later gates join the open tile pass, so a depth-20
    random circuit needs far fewer full-state passes than cutting the reordered list in runs;
    the partition stays a sequence of consecutive runs of the execution order."""
    c = wc.rqc(30, 20, seed=3)
    monkeypatch.setenv("QGPU_PASS_SCHED", "0")  # the lookahead alone (the pass scheduler ignores it)

    def traffic(la):
        monkeypatch.setenv("QGPU_LOOKAHEAD", str(la))
        plan = q.Circuit(c.qasm()).plan(c.n, 1, 2, 12)
        pos = 0
        for first, count, *_ in plan:
            assert first == pos
            pos += count
        return sum(2.0 ** r[3] + 2.0 ** r[4] for r in plan if r[2] == 0) / 2 ** (c.n + 1)

    assert traffic(192) < 0.6 * traffic(0)
