"""GPU parity of the GFC compression kernels (csrc/gfc.cu) against the oracle (oracle/gfc.py):
byte-exact streams and offsets on the golden cases, random bit patterns, ragged sizes and
simulated states; lossless round trips at large sizes with sampled segments checked against
the oracle one by one. All calls go through the C ABI (qgpu_gfc_*)."""
import json
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden", "gfc_examples.json")


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu
    from oracle import gfc
    assert torch.cuda.is_available()
    qgpu.load()
    return torch, qgpu, gfc


def gpu_compress(env, x: np.ndarray, seg: int):
    torch, qgpu, _ = env
    words = np.ascontiguousarray(x).view(np.uint64).ravel()
    n = words.size
    d_in = torch.from_numpy(words.view(np.int64).copy()).cuda()
    cap = qgpu.gfc_max_bytes(n, seg)
    d_out = torch.zeros(max(cap, 16), dtype=torch.uint8, device="cuda")
    nseg = (n + seg - 1) // seg
    d_off = torch.zeros(nseg + 1, dtype=torch.int64, device="cuda")
    nb = qgpu.gfc_compress(d_in.data_ptr(), n, seg, d_out.data_ptr(), cap, d_off.data_ptr())
    stream = d_out[:nb].cpu().numpy().tobytes()
    off = d_off.cpu().numpy().view(np.uint64)
    # decompress on the device and compare every bit pattern
    d_back = torch.empty(max(n, 1), dtype=torch.int64, device="cuda")
    qgpu.gfc_decompress(d_out.data_ptr(), d_off.data_ptr(), n, seg, d_back.data_ptr())
    torch.cuda.synchronize()
    back = d_back[:n].cpu().numpy().view(np.uint64)
    assert np.array_equal(back, words), "GPU round trip is not lossless"
    return stream, off


def test_golden_cases(env):
    _, _, gfc = env
    for case in json.load(open(GOLD))["cases"]:
        words = np.array([int(h, 16) for h in case["words_hex"]], dtype=np.uint64)
        want = b"".join(bytes.fromhex(h) * r for h, r in case["stream_parts"])
        stream, off = gpu_compress(env, words, case["seg_len"])
        assert stream == want, case["name"]
        assert off.tolist() == case["offsets"]


@pytest.mark.parametrize("n,seg", [(1, 32), (31, 32), (33, 32), (1000, 96), (5000, 1024), (70001, 4096)])
def test_random_bits_vs_oracle(env, n, seg):
    _, _, gfc = env
    rng = np.random.default_rng(n + seg)
    # a mix: random patterns, small perturbations (compressible), special values
    base = rng.integers(0, 2 ** 62, size=n, dtype=np.uint64)
    small = rng.integers(0, 4096, size=n, dtype=np.uint64)
    pick = rng.integers(0, 3, size=n)
    words = np.where(pick == 0, base, np.where(pick == 1, np.uint64(0x3FE0000000000000) + small,
                                                np.uint64(0x8000000000000000)))
    stream, off = gpu_compress(env, words.astype(np.uint64), seg)
    ws, wo = gfc.compress(words.astype(np.uint64).view(np.float64), seg)
    assert off.tolist() == wo.tolist()
    assert stream == ws


def test_simulated_states_vs_oracle(env):
    _, _, gfc = env
    from oracle import statevector as sv
    from workloads import circuits as wc
    for c in (wc.qaoa(12, 2, seed=1), wc.iqp(12), wc.qft(12, x=37), wc.gs(3, 4), wc.qft(12)):
        psi = sv.simulate(c.qasm())
        stream, off = gpu_compress(env, psi, 1024)
        ws, wo = gfc.compress(psi, 1024)
        assert off.tolist() == wo.tolist() and stream == ws


def test_large_state_sampled_segments(env):
    """2^23 doubles (a 22-qubit QAOA state from the library itself): lossless on the device, and
    sampled segments byte-identical to the oracle's encoding of the same segment."""
    torch, qgpu, gfc = env
    from workloads import circuits as wc
    n_q = 22
    with qgpu.State(n_q) as s:
        s.apply_circuit(qgpu.Circuit(wc.qaoa(n_q, 2, seed=1).qasm()))
        psi = s.amplitudes()
    seg = 4096
    stream, off = gpu_compress(env, psi, seg)
    words = psi.view(np.float64)
    rng = np.random.default_rng(3)
    nseg = len(off) - 1
    for sidx in list(rng.integers(0, nseg, size=6)) + [0, nseg - 1]:
        ref = gfc.encode_segment(gfc.as_words(words[sidx * seg:(sidx + 1) * seg]))
        assert stream[int(off[sidx]):int(off[sidx + 1])] == ref


def test_errors(env):
    torch, qgpu, _ = env
    d_in = torch.zeros(64, dtype=torch.float64, device="cuda")
    d_out = torch.zeros(16, dtype=torch.uint8, device="cuda")
    d_off = torch.zeros(2, dtype=torch.int64, device="cuda")
    with pytest.raises(qgpu.QgpuError):
        qgpu.gfc_compress(d_in.data_ptr(), 64, 48, d_out.data_ptr(), 16, d_off.data_ptr())
    with pytest.raises(qgpu.QgpuError):  # 64 zeros need 96 bytes
        qgpu.gfc_compress(d_in.data_ptr(), 64, 64, d_out.data_ptr(), 16, d_off.data_ptr())
    assert qgpu.gfc_compress(d_in.data_ptr(), 0, 64, d_out.data_ptr(), 16, d_off.data_ptr()) == 0
