"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element.

Tolerances (north star / DESIGN.md §6): max |delta| <= 1e-10 on amplitudes, |1 - sum|psi|^2|
<= 1e-12, pruning bitmap and schedule bit-exact, prune on/off exactly equal."""
import math

import numpy as np
import pytest

from oracle import qasm as oq
from oracle import schedule as osch
from oracle import statevector as osv
from workloads import circuits as wc

pytestmark = pytest.mark.gpu

TOL = 1e-10
NORM_TOL = 1e-12


@pytest.fixture(scope="module")
def q():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


def gpu_run(q, text, n=None, **cfg):
    c = q.Circuit(text)
    nn = n or c.info()[0]
    with q.State(nn, **cfg) as s:
        s.apply_circuit(c)
        return s.amplitudes()


def oracle_run(text):
    return osv.simulate(text)


CFGS = [dict(fuse_bits=0, reorder=0), dict(fuse_bits=0, reorder=2), dict(fuse_bits=12, reorder=2),
        dict(fuse_bits=7, reorder=1), dict(fuse_bits=9, reorder=0), dict(fuse_bits=12, prune=0)]


@pytest.mark.parametrize("cfg", CFGS, ids=lambda d: "-".join(f"{k}{v}" for k, v in d.items()))
def test_c1_ghz_qft5(q, cfg):
    text = wc.ghz_qft(5).qasm()
    got = gpu_run(q, text, **cfg)
    ref = oracle_run(text)
    assert np.abs(got - ref).max() <= TOL
    y = np.arange(32)
    assert np.abs(got - (1 + np.exp(2j * np.pi * 31 * y / 32)) / 8).max() <= TOL
    assert abs(1 - np.vdot(got, got).real) <= NORM_TOL


FUZZ = [(6, 80, 1), (9, 200, 2), (11, 300, 3), (13, 300, 4), (14, 400, 5), (16, 300, 6)]


@pytest.mark.parametrize("n,G,seed", FUZZ)
@pytest.mark.parametrize("cfg", CFGS, ids=lambda d: "-".join(f"{k}{v}" for k, v in d.items()))
def test_random_circuit_fuzz(q, n, G, seed, cfg):
    text = wc.random_circuit(n, G, seed=seed).qasm()
    got = gpu_run(q, text, **cfg)
    ref = oracle_run(text)
    assert np.abs(got - ref).max() <= TOL
    assert abs(1 - np.vdot(got, got).real) <= NORM_TOL


@pytest.mark.parametrize("fam", ["qft", "qaoa", "rqc", "gs", "hlf", "iqp", "bv", "grqc"])
@pytest.mark.parametrize("fuse", [0, 12])
def test_families_vs_oracle(q, fam, fuse):
    c = {"qft": lambda: wc.qft(18, x=12345), "qaoa": lambda: wc.qaoa(16, 2, seed=1),
         "rqc": lambda: wc.rqc(18, 12, seed=3), "gs": lambda: wc.gs(4, 4),
         "hlf": lambda: wc.hlf(4, 4, seed=2), "iqp": lambda: wc.iqp(14),
         "bv": lambda: wc.bv(15, 0b101101110110101),
         "grqc": lambda: wc.grqc(4, 4, 60, seed=5)}[fam]()
    text = c.qasm()
    got = gpu_run(q, text, fuse_bits=fuse)
    ref = oracle_run(text)
    assert np.abs(got - ref).max() <= TOL


def _rand_state(n, seed):
    r = np.random.default_rng(seed)
    v = r.normal(size=1 << n) + 1j * r.normal(size=1 << n)
    return v / np.linalg.norm(v)


@pytest.mark.parametrize("n", [6, 12, 19])
def test_single_gates_every_position(q, n):
    """a6/a7/a8 kernels on a fully involved random state: every target position (lane bits
    use the shuffle path, higher bits the two-stream path), with and without controls."""
    rng = np.random.default_rng(n)
    psi0 = _rand_state(n, n)
    ref = psi0.copy()
    with q.State(n) as s:
        s.set_amplitudes(psi0)
        for t in range(n):
            U = oq.u3(*rng.uniform(-3, 3, 3))
            s.apply_gate(U, [t]); osv.apply_gate(ref, n, U, [t])
            c = int((t + 1 + rng.integers(0, n - 1)) % n)
            s.apply_gate(U, [t], [c]); osv.apply_gate(ref, n, U, [t], [c])
            t2 = int((t + 3) % n)
            if t2 != t:
                U2 = np.linalg.qr(rng.normal(size=(4, 4)) + 1j * rng.normal(size=(4, 4)))[0]
                s.apply_gate(U2, [t, t2]); osv.apply_gate(ref, n, U2, [t, t2])
                D = np.diag(np.exp(1j * rng.uniform(-3, 3, 4)))
                s.apply_gate(D, [t2, t]); osv.apply_gate(ref, n, D, [t2, t])
            s.apply_gate(oq.phase(0.3), [t], [(t + 2) % n]); osv.apply_gate(ref, n, oq.phase(0.3), [t], [(t + 2) % n])
        got = s.amplitudes()
    assert np.abs(got - ref).max() <= TOL


@pytest.mark.parametrize("seed", range(4))
def test_apply_gate_stream_bitmap_and_expand(q, seed):
    """Gate-by-gate API from |0..0>: first-touch expansion, pruning bitmap bit-exact after
    every gate, data zero-map soundness, and amplitudes vs oracle."""
    n = 12
    c = wc.random_circuit(n, 60, seed=100 + seed)
    _, gates = oq.parse(c.qasm())
    ref = osv.zero_state(n)
    inv = 0
    with q.State(n) as s:
        for k, g in enumerate(gates):
            s.apply_gate(g.U, list(g.targets), list(g.controls))
            osv.apply_gate(ref, n, g.U, g.targets, g.controls)
            inv = osch.update_involvement(inv, g.qubits)
            assert s.involvement() == inv
            for cb in (0, 3, 7):
                bm = s.chunk_bitmap(cb)
                assert list(bm) == osch.chunk_bitmap(inv, n, cb)
            if k % 10 == 9:
                got = s.amplitudes()
                assert np.abs(got - ref).max() <= TOL
                z = osv.zero_map(got, n, 3)
                assert np.all(z[~np.array(osch.chunk_bitmap(inv, n, 3), dtype=bool)])
        order, invs = s.schedule()
    assert list(order) == list(range(len(gates)))
    assert [int(x) for x in invs] == osch.involvement_trace(gates)


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_circuit_schedule_trace_exact(q, mode):
    """qgpu_get_schedule equals the oracle's Alg.2/Alg.3 replay and involvement trace."""
    c = wc.qaoa(12, 2, seed=7)
    text = c.qasm()
    _, gates = oq.parse(text)
    with q.State(12, reorder=mode) as s:
        s.apply_circuit(q.Circuit(text))
        order, invs = s.schedule()
        st = s.stats()
    ref = osch.reorder(gates, mode)
    assert list(order) == ref
    assert [int(x) for x in invs] == osch.involvement_trace(gates, ref)
    assert st["ops_before_full_involvement"] == osch.ops_before_full_involvement(gates, 12, ref)


@pytest.mark.parametrize("fuse", [0, 9, 12])
def test_pruning_neutrality_exact(q, fuse):
    """P:221 / SURVEY §8c-P14: prune=1 and prune=0 give exactly equal amplitudes."""
    text = wc.random_circuit(15, 250, seed=21).qasm()
    a = gpu_run(q, text, fuse_bits=fuse, prune=1)
    b = gpu_run(q, text, fuse_bits=fuse, prune=0)
    assert np.array_equal(a, b)


def test_pruning_skips_chunks(q):
    """Pruning measurably skips zero chunks: processed amplitudes < unpruned on QFT."""
    text = wc.qft(20).qasm()
    with q.State(20, chunk_bits=10) as s:
        s.apply_circuit(q.Circuit(text))
        st = s.stats()
    assert st["chunks_skipped"] > 0
    assert st["amps_processed"] < st["amps_full"]


@pytest.mark.parametrize("n,x", [(20, 0), (20, 777777), (22, 1234567)])
def test_qft_closed_form(q, n, x):
    text = wc.qft(n, x=x).qasm()
    got = gpu_run(q, text)
    y = np.arange(1 << n)
    exp = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / math.sqrt(1 << n)
    assert np.abs(got - exp).max() <= TOL


def test_graph_state_and_hlf_closed_form(q):
    c = wc.gs(4, 5)
    got = gpu_run(q, c.qasm())
    xs = np.arange(1 << c.n)
    par = np.zeros(1 << c.n, dtype=np.int64)
    for u, v in c.meta["edges"]:
        par ^= ((xs >> u) & 1) & ((xs >> v) & 1)
    assert np.abs(got - (1 - 2 * par) / math.sqrt(1 << c.n)).max() <= TOL
    from test_oracle_pins import hlf_expected_probabilities
    h = wc.hlf(4, 4, seed=3)
    c = q.Circuit(h.qasm())
    with q.State(h.n) as s:
        s.apply_circuit(c)
        p = s.probabilities(list(range(h.n)))
    assert np.abs(p - hlf_expected_probabilities(h.n, h.meta["edges"], h.meta["s"])).max() <= 1e-12


@pytest.mark.parametrize("n,w,k", [(8, 77, 3), (12, 3000, 10)])
def test_grover_mcz(q, n, w, k):
    """MCZ with n-1 controls through qgpu_apply_gate."""
    X, H, Z = oq.X, oq.H, oq.Z
    full = (1 << n) - 1
    with q.State(n, fuse_bits=0) as s:
        def xs(mask):
            for b in range(n):
                if mask >> b & 1:
                    s.apply_gate(X, [b])
        for b in range(n):
            s.apply_gate(H, [b])
        for _ in range(k):
            xs(full & ~w); s.apply_gate(Z, [n - 1], list(range(n - 1))); xs(full & ~w)
            for b in range(n):
                s.apply_gate(H, [b])
            xs(full); s.apply_gate(Z, [n - 1], list(range(n - 1))); xs(full)
            for b in range(n):
                s.apply_gate(H, [b])
        p = s.probabilities(list(range(n)))
    th = math.asin(2 ** (-n / 2))
    assert abs(p[w] - math.sin((2 * k + 1) * th) ** 2) <= 1e-12
    assert abs(p.sum() - 1) <= NORM_TOL


def test_probabilities_vs_oracle(q):
    n = 14
    text = wc.random_circuit(n, 200, seed=31).qasm()
    ref = oracle_run(text)
    c = q.Circuit(text)
    with q.State(n) as s:
        s.apply_circuit(c)
        for qs in ([], [0], [13, 2], [5, 9, 1, 11], list(range(n)), list(range(n))[::-1]):
            p = s.probabilities(qs)
            assert np.abs(p - osv.probabilities(ref, n, qs)).max() <= 1e-12


@pytest.mark.parametrize("hist", [0, 1])
def test_probabilities_mapped_and_histogram_kernels(q, hist, monkeypatch):
    """Both readout kernels (mapped: requested positions dealt to lanes/warps/CTAs; histogram:
    QGPU_PROBS_HIST=1) on fully and partially involved states, many qubit subsets."""
    if hist:
        monkeypatch.setenv("QGPU_PROBS_HIST", "1")
    rng = np.random.default_rng(77)
    n = 16
    for nq_involved in (16, 11):
        c = wc.random_circuit(nq_involved, 160, seed=40 + nq_involved)
        text = c.qasm().replace(f"qreg q[{nq_involved}];", f"qreg q[{n}];")
        ref = oracle_run(text)
        with q.State(n) as s:
            s.apply_circuit(q.Circuit(text))
            subsets = [[], [0], list(range(n)), [15, 3], list(range(10)), list(range(6, 16))]
            subsets += [list(rng.choice(n, size=int(rng.integers(1, 13)), replace=False)) for _ in range(10)]
            for qs in subsets:
                qs = [int(x) for x in qs]
                p = s.probabilities(qs)
                assert np.abs(p - osv.probabilities(ref, n, qs)).max() <= 1e-12, qs


def test_bv_large(q):
    n, sec = 24, 0b10110011100011110000101
    with q.State(n) as s:
        s.apply_circuit(q.Circuit(wc.bv(n, sec).qasm()))
        p = s.probabilities(list(range(n - 1)))
    assert abs(p[sec] - 1) <= 1e-12


@pytest.mark.parametrize("fam", ["rqc", "qaoa"])
def test_mirror_returns_to_zero(q, fam):
    c = {"rqc": lambda: wc.rqc(24, 10, seed=3), "qaoa": lambda: wc.qaoa(24, 2, seed=1)}[fam]()
    m = wc.mirror(c)
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(m.qasm()))
        a = s.amplitudes(0, 1024)
        p = s.probabilities([])
    assert abs(a[0] - 1) <= TOL and np.abs(a[1:]).max() <= TOL
    assert abs(p[0] - 1) <= NORM_TOL


def test_errors(q):
    with q.State(8) as s:
        with pytest.raises(q.QgpuError) as e:
            s.apply_gate(oq.H, [8])
        assert e.value.kind == "INVALID_ARG"
        with pytest.raises(q.QgpuError):
            s.apply_gate(oq.H, [1], [1])
        with pytest.raises(q.QgpuError):
            s.probabilities([0, 0])
        big = q.Circuit(wc.qft(9).qasm())
        with pytest.raises(q.QgpuError):
            s.apply_circuit(big)
        s.apply_gate(oq.H, [0])  # still usable
        assert abs(s.amplitudes(0, 2)[1] - 1 / math.sqrt(2)) <= TOL


def test_torch_buffer_and_stream(q):
    """PyTorch supplies device memory and the stream (plumbing only)."""
    import torch
    n = 16
    buf = torch.empty(2 << n, dtype=torch.float64, device="cuda")
    stream = torch.cuda.Stream()
    text = wc.qft(n, x=999).qasm()
    with q.State(n, state_buffer=buf.data_ptr(), state_buffer_bytes=buf.numel() * 8,
                 stream=stream.cuda_stream) as s:
        s.apply_circuit(q.Circuit(text))
        s.synchronize()
        got = torch.view_as_complex(buf.view(-1, 2)).cpu().numpy()
        pos = s.qubit_map()
    # the buffer is in physical order; map back to logical through the qubit map
    ref = oracle_run(text)
    idx = np.zeros(1 << n, dtype=np.int64)
    xs = np.arange(1 << n)
    for lq, p in enumerate(pos):
        idx |= ((xs >> lq) & 1) << p
    assert np.abs(got[idx] - ref).max() <= TOL


# ----------------------------------------------------------------------------- JIT path
JIT_CIRCS = {
    "fuzz12": lambda: wc.random_circuit(12, 300, seed=41),
    "fuzz14": lambda: wc.random_circuit(14, 300, seed=42),
    "qft16x": lambda: wc.qft(16, x=4321),
    "qaoa14": lambda: wc.qaoa(14, 2, seed=1),
    "rqc14": lambda: wc.rqc(14, 10, seed=3),
    "hlf4x4": lambda: wc.hlf(4, 4, seed=2),
}


@pytest.mark.parametrize("name", sorted(JIT_CIRCS))
@pytest.mark.parametrize("fuse", [9, 12])
def test_jit_specialised_kernels_vs_oracle(q, name, fuse):
    """jit=2: every fused pass runs an NVRTC-specialised kernel; parity vs the oracle and
    agreement with the interpreted tile kernel (jit=0)."""
    c = JIT_CIRCS[name]()
    text = c.qasm()
    qc = q.Circuit(text)
    with q.State(c.n, fuse_bits=fuse, jit=2) as s:
        s.apply_circuit(qc)
        got = s.amplitudes()
        st = s.stats()
    assert st["jit_launches"] > 0
    ref = oracle_run(text)
    assert np.abs(got - ref).max() <= TOL
    interp = gpu_run(q, text, fuse_bits=fuse, jit=0)
    assert np.abs(got - interp).max() <= 1e-13


def test_jit_pruning_neutrality_exact(q):
    text = wc.random_circuit(15, 250, seed=21).qasm()
    a = gpu_run(q, text, fuse_bits=12, prune=1, jit=2)
    b = gpu_run(q, text, fuse_bits=12, prune=0, jit=2)
    assert np.array_equal(a, b)


SCHED_CIRCS = {
    "qaoa": lambda: wc.qaoa(20, 2, seed=5),
    "hlf": lambda: wc.hlf(4, 5, seed=3),
    "rqc": lambda: wc.rqc(18, 8, seed=4),
    "randdiag": lambda: wc.random_circuit(16, 240, seed=21, names=["cp", "cz", "rz", "cx", "crx", "ccx", "t",
                                                                     "h", "rzz", "x", "u1", "crz", "s", "sx"]),
}


@pytest.mark.parametrize("name", sorted(SCHED_CIRCS))
@pytest.mark.parametrize("sched", ["0", "2"])
@pytest.mark.parametrize("reorder", ["1", "0"])
def test_pass_schedule_and_op_clustering_vs_oracle(q, name, sched, reorder, monkeypatch):
    """The pass-aware execution order forced on (QGPU_PASS_SCHED=2) and off (0), each with the
    intra-pass op clustering on and off (QGPU_PASS_REORDER), on the NVRTC kernels at the
    library's default threshold: every amplitude against the oracle (commuting
    reorders change rounding only)."""
    monkeypatch.setenv("QGPU_PASS_SCHED", sched)
    monkeypatch.setenv("QGPU_PASS_REORDER", reorder)
    monkeypatch.setenv("QGPU_JIT_MIN_BITS", "12")
    c = SCHED_CIRCS[name]()
    got = gpu_run(q, c.qasm())
    ref = oracle_run(c.qasm())
    assert np.abs(got - ref).max() <= TOL
    assert abs(1.0 - float(np.sum(np.abs(got) ** 2))) <= NORM_TOL
