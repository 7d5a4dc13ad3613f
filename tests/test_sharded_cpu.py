"""Sharded (multi-GPU) protocol on CPU: world_size 2 and 4 with the gloo backend.

The library's host planner (qgpu_circuit_plan_text: physical gates, rank activation, global-local
swap passes) is executed here by an independent numpy shard executor, one process per rank, with
the swaps done as torch.distributed send/recv over gloo. The gathered state, mapped back through
the final qubit map, must equal the oracle. This covers the N>1 host logic (a10) without GPUs.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import statevector as osv
from workloads import circuits as wc


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _parse_plan(text):
    passes, final_map = [], None
    for line in text.strip().splitlines():
        w = line.split()
        if w[0] == "P":
            kind, kin, kout, kg, kgf, nsw = map(int, w[1:7])
            sw = [(int(w[7 + 2 * i]), int(w[8 + 2 * i])) for i in range(nsw)]
            passes.append({"kind": kind, "kg": kg, "kg_from": kgf, "swaps": sw, "gates": []})
        elif w[0] == "G":
            nt, p0, p1, pc, diag = int(w[1]), int(w[2]), int(w[3]), int(w[4]), int(w[5])
            vals = list(map(float, w[6:]))
            d = 1 << nt
            U = np.array(vals[0::2], dtype=float) + 1j * np.array(vals[1::2], dtype=float)
            passes[-1]["gates"].append((nt, [p0, p1][:nt], pc, bool(diag), U.reshape(d, d)))
        elif w[0] == "M":
            final_map = [int(x) for x in w[1:]]
    return passes, final_map


def _apply(psi, rank, m, nt, targets, pc, U):
    """Apply one gate to this rank's shard; index bits >= m are this rank's bits."""
    L = psi.size
    gidx = (np.uint64(rank) << np.uint64(m)) | np.arange(L, dtype=np.uint64)
    ok = (gidx & np.uint64(pc)) == np.uint64(pc)
    tmask = 0
    for t in targets:
        tmask |= 1 << t
    if all(t < m for t in targets):
        base = np.nonzero(ok & ((gidx & np.uint64(tmask)) == 0))[0]
        offs = []
        for j in range(1 << nt):
            o = 0
            for k in range(nt):
                if (j >> k) & 1:
                    o |= 1 << targets[k]
            offs.append(o)
        v = np.stack([psi[base + o] for o in offs])
        w = U @ v
        for j, o in enumerate(offs):
            psi[base + o] = w[j]
    else:  # only diagonal gates may have a target on a rank bit
        assert np.all(U == np.diag(np.diag(U)))
        sel = np.zeros(L, dtype=np.int64)
        for k, t in enumerate(targets):
            sel |= ((gidx >> np.uint64(t)) & np.uint64(1)).astype(np.int64) << k
        f = np.where(ok, np.diag(U)[sel], 1.0)
        psi *= f


def _shard_main(rank, world, port, text, n, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = world.bit_length() - 1
    m = n - g
    psi = np.zeros(1 << m, dtype=np.complex128)
    if rank == 0:
        psi[0] = 1.0
    passes, fmap = _parse_plan(text)
    loc = np.arange(psi.size)
    for p in passes:
        if p["kind"] == 6 and p["kg_from"] < 0:  # cross-rank expand: copy of rank r - 2^kg_from
            kf, kg = -1 - p["kg_from"], p["kg"]
            assert kg == kf + 1
            lo = 1 << kf
            if rank < lo and rank + lo < (1 << kg):
                dist.send(torch.from_numpy(psi.view(np.float64).copy()), rank + lo)
            elif lo <= rank < (1 << kg):
                buf = torch.empty(2 * psi.size, dtype=torch.float64)
                dist.recv(buf, rank - lo)
                psi[:] = buf.numpy().view(np.complex128)
        if p["kind"] == 5 and rank < (1 << p["kg"]):
            # ONE batched swap: for every pair (g_i, l_i) the logical qubit on rank bit g_i - m
            # trades places with the one on local position l_i. The amplitude at (rank r, local i)
            # moves to the rank whose bits g_i - m equal i's bits l_i, at the local index whose
            # bits l_i equal r's bits g_i - m (the rest of i unchanged): an all-to-all inside each
            # group of ranks that differ only in the swapped rank bits.
            pairs = p["swaps"]
            dest_rank = np.full(psi.size, rank, dtype=np.int64)
            dest_loc = loc.copy()
            for gp, lp in pairs:
                j = gp - m
                bit_l = (loc >> lp) & 1
                dest_rank = (dest_rank & ~(1 << j)) | (bit_l << j)
                dest_loc = (dest_loc & ~(1 << lp)) | (((rank >> j) & 1) << lp)
            peers = sorted(set(dest_rank.tolist()))
            new = psi.copy()
            mine = dest_rank == rank
            new[dest_loc[mine]] = psi[mine]
            reqs, bufs = [], {}
            for pr in peers:
                if pr == rank:
                    continue
                sel = dest_rank == pr
                send = torch.from_numpy(np.ascontiguousarray(
                    np.stack([dest_loc[sel].astype(np.float64), psi[sel].real, psi[sel].imag])).copy())
                bufs[pr] = torch.empty_like(send)
                reqs.append(dist.isend(send, pr))
                reqs.append(dist.irecv(bufs[pr], pr))
            for r_ in reqs:
                r_.wait()
            for pr, b in bufs.items():
                a = b.numpy()
                new[a[0].astype(np.int64)] = a[1] + 1j * a[2]
            psi = new
        for (nt, targets, pc, diag, U) in p["gates"]:
            _apply(psi, rank, m, nt, targets, pc, U)
    t = torch.from_numpy(psi.view(np.float64).copy())
    gathered = [torch.empty_like(t) for _ in range(world)] if rank == 0 else None
    dist.gather(t, gathered, dst=0)
    if rank == 0:
        full = np.concatenate([x.numpy().view(np.complex128) for x in gathered])
        out.put((full.tobytes(), fmap))
    dist.barrier()
    dist.destroy_process_group()


def _run_sharded(q, circ, world, fuse, mode=2):
    text = q.Circuit(circ.qasm()).plan_text(circ.n, world, mode, fuse)
    ctx = mp.get_context("spawn")
    out = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_main, args=(r, world, port, text, circ.n, out)) for r in range(world)]
    for p in procs:
        p.start()
    full_bytes, fmap = out.get()
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    full = np.frombuffer(full_bytes, dtype=np.complex128)
    n = circ.n
    xs = np.arange(1 << n)
    phys = np.zeros(1 << n, dtype=np.int64)
    never = np.zeros(1 << n, dtype=bool)
    for lq, pos in enumerate(fmap):
        bit = (xs >> lq) & 1
        if pos < 0:
            never |= bit.astype(bool)
        else:
            phys |= bit << pos
    logical = np.where(never, 0, full[phys])
    return logical, text


@pytest.fixture(scope="module")
def q():
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("name", ["random", "qft", "rqc", "ghz", "grqc"])
def test_sharded_protocol_vs_oracle(q, world, name):
    c = {"random": lambda: wc.random_circuit(8, 90, seed=world),
         "qft": lambda: wc.qft(8, x=171),
         "rqc": lambda: wc.rqc(8, 6, seed=3),
         "ghz": lambda: wc.ghz(9),
         "grqc": lambda: wc.grqc(2, 4, 40, seed=5)}[name]()
    got, text = _run_sharded(q, c, world, fuse=12)
    ref = osv.simulate(c.qasm())
    assert np.abs(got - ref).max() <= 1e-12
    if name in ("random", "rqc", "ghz"):
        assert "\nP 5 " in "\n" + text  # the plan exercised at least one global-local swap


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("name", ["random", "qft", "rqc", "gs", "hlf"])
def test_sharded_protocol_early_global_placement(q, world, name, monkeypatch):
    """§8e cross-rank first-touch expand: with QGPU_GLOBAL_MIN_LOCAL=2 the first log2 G qubits
    first touched by an uncontrolled 1-qubit gate go to rank bits while only 2 local positions
    are assigned (copy activations), so later non-diagonal gates on them need batched swaps with
    few assigned local positions; executed with gloo against the oracle."""
    monkeypatch.setenv("QGPU_GLOBAL_MIN_LOCAL", "2")
    c = {"random": lambda: wc.random_circuit(8, 90, seed=world + 10),
         "qft": lambda: wc.qft(8, x=171),
         "rqc": lambda: wc.rqc(8, 6, seed=3),
         "gs": lambda: wc.gs(2, 4),
         "hlf": lambda: wc.hlf(2, 4, seed=2)}[name]()
    got, text = _run_sharded(q, c, world, fuse=12)
    assert np.abs(got - osv.simulate(c.qasm())).max() <= 1e-12
    lines = text.splitlines()
    assert any(l.startswith("P 6 ") and int(l.split()[5]) < 0 for l in lines)  # a copy activation


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("name", ["qft0", "randdiag"])
def test_sharded_protocol_refined_rule(q, world, name):
    """NEXT-1 plans (reorder mode 2 + 4) through the same shard executor: skipped and restricted
    gates, rank-bit diagonal restrictions and swaps stay exact."""
    c = {"qft0": lambda: wc.qft(8),
         "randdiag": lambda: wc.random_circuit(8, 90, seed=5, names=["cp", "cz", "rz", "cx", "crx", "ccx",
                                                                      "h", "rzz", "x", "crz", "swap"])}[name]()
    got, text = _run_sharded(q, c, world, fuse=12, mode=6)
    assert np.abs(got - osv.simulate(c.qasm())).max() <= 1e-12

