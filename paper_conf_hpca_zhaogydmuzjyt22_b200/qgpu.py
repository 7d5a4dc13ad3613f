"""Thin ctypes binding of libqgpu.so (include/qgpu.h): argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels. If the shared library is
missing the import fails loudly -- there is no CPU fallback. PyTorch, when used by the caller,
only supplies device memory (``state_buffer``) and the stream.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libqgpu.so")

QGPU_OK = 0
STATUS = {0: "OK", 1: "INVALID_ARG", 2: "OUT_OF_MEMORY", 3: "UNSUPPORTED", 4: "PARSE",
          5: "CUDA", 6: "NCCL", 7: "STATE"}

EXPORTS = [
    "qgpu_config_init", "qgpu_state_create", "qgpu_state_destroy", "qgpu_state_reset",
    "qgpu_set_amplitudes", "qgpu_synchronize", "qgpu_state_info", "qgpu_apply_gate",
    "qgpu_apply_circuit", "qgpu_apply_circuit_probabilities", "qgpu_get_amplitudes", "qgpu_get_amplitudes_device",
    "qgpu_probabilities", "qgpu_circuit_from_qasm", "qgpu_circuit_info", "qgpu_circuit_destroy",
    "qgpu_circuit_reorder", "qgpu_circuit_plan", "qgpu_circuit_plan_text", "qgpu_circuit_jit_check", "qgpu_get_involvement", "qgpu_get_chunk_bitmap",
    "qgpu_get_schedule", "qgpu_get_qubit_map", "qgpu_get_stats", "qgpu_reset_stats",
    "qgpu_nccl_unique_id", "qgpu_gfc_max_bytes", "qgpu_gfc_compress", "qgpu_gfc_decompress",
    "qgpu_last_error", "qgpu_version", "qgpu_get_pass_profile", "qgpu_measure_fp64_peak",
    "qgpu_set_timing",
]


class QgpuError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"qgpu {STATUS.get(status, status)}: {msg}")
        self.status = status
        self.kind = STATUS.get(status, str(status))


class Config(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_uint32), ("device", ctypes.c_int), ("stream", ctypes.c_void_p),
        ("state_buffer", ctypes.c_void_p), ("state_buffer_bytes", ctypes.c_uint64),
        ("rank", ctypes.c_int), ("world_size", ctypes.c_int), ("nccl_unique_id", ctypes.c_void_p),
        ("chunk_bits", ctypes.c_int), ("prune", ctypes.c_int), ("reorder", ctypes.c_int),
        ("fuse_bits", ctypes.c_int), ("timing", ctypes.c_int), ("swap_slab_bytes", ctypes.c_uint64),
        ("jit", ctypes.c_int), ("host_slice_bits", ctypes.c_int), ("involve_rule", ctypes.c_int),
        ("host_compress", ctypes.c_int),
    ]


class Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "gates_applied", "passes", "kernels_launched", "relabels", "amps_processed", "amps_full",
        "chunks_processed", "chunks_skipped", "algo_bytes", "unfused_bytes", "swaps", "swap_bytes")] + [
        ("ops_before_full_involvement", ctypes.c_int64), ("kernel_ms", ctypes.c_double),
        ("tile_kernel_ms", ctypes.c_double), ("tile_kernel_launches", ctypes.c_uint64),
        ("tile_algo_bytes", ctypes.c_uint64), ("swap_ms", ctypes.c_double),
        ("h2d_bytes", ctypes.c_uint64), ("d2h_bytes", ctypes.c_uint64),
        ("jit_launches", ctypes.c_uint64), ("jit_compiles", ctypes.c_uint64), ("jit_ms", ctypes.c_double),
        ("host_h2d_bytes", ctypes.c_uint64), ("host_d2h_bytes", ctypes.c_uint64),
        ("host_slice_loads", ctypes.c_uint64), ("host_slice_skips", ctypes.c_uint64),
        ("host_runs", ctypes.c_uint64), ("host_ms", ctypes.c_double), ("swap_bits", ctypes.c_uint64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class PassProfile(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("k_in", ctypes.c_int32), ("k_out", ctypes.c_int32),
                ("n_gates", ctypes.c_int32), ("ms", ctypes.c_double), ("bytes", ctypes.c_uint64),
                ("amps_computed", ctypes.c_uint64), ("fp64_ops", ctypes.c_double),
                ("lane_ops", ctypes.c_int32), ("remaps", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libqgpu.so (raises if it has not been built: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run `python -m paper_conf_hpca_zhaogydmuzjyt22_b200.build`")
    lib = ctypes.CDLL(path)
    P, I, U64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64
    sig = {
        "qgpu_config_init": [P], "qgpu_state_create": [I, P, P], "qgpu_state_destroy": [P],
        "qgpu_state_reset": [P], "qgpu_set_amplitudes": [P, P], "qgpu_synchronize": [P],
        "qgpu_state_info": [P, P, P, P], "qgpu_apply_gate": [P, P, I, P, I, P],
        "qgpu_apply_circuit": [P, P], "qgpu_apply_circuit_probabilities": [P, P, I, P, P],
        "qgpu_get_amplitudes": [P, U64, U64, P],
        "qgpu_get_amplitudes_device": [P, U64, U64, P], "qgpu_probabilities": [P, I, P, P],
        "qgpu_circuit_from_qasm": [ctypes.c_char_p, ctypes.c_size_t, P],
        "qgpu_circuit_info": [P, P, P], "qgpu_circuit_destroy": [P],
        "qgpu_circuit_reorder": [P, I, P, U64, P], "qgpu_circuit_plan": [P, I, I, I, I, P, U64, P],
        "qgpu_circuit_jit_check": [P, I, I, I, P],
        "qgpu_circuit_plan_text": [P, I, I, I, I, P, ctypes.c_size_t, P],
        "qgpu_get_involvement": [P, P], "qgpu_get_chunk_bitmap": [P, I, P, U64],
        "qgpu_get_schedule": [P, P, P, U64, P], "qgpu_get_qubit_map": [P, P],
        "qgpu_get_stats": [P, P], "qgpu_reset_stats": [P],
        "qgpu_nccl_unique_id": [P, ctypes.c_size_t],
        "qgpu_gfc_max_bytes": [U64, ctypes.c_uint32, P],
        "qgpu_gfc_compress": [P, U64, ctypes.c_uint32, P, U64, P, P, P],
        "qgpu_gfc_decompress": [P, P, U64, ctypes.c_uint32, P, P],
        "qgpu_get_pass_profile": [P, P, U64, P], "qgpu_measure_fp64_peak": [I, P],
        "qgpu_set_timing": [P, I],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    lib.qgpu_last_error.restype = ctypes.c_char_p
    lib.qgpu_last_error.argtypes = []
    lib.qgpu_version.restype = ctypes.c_char_p
    lib.qgpu_version.argtypes = []
    _lib = lib
    return lib


def _check(rc: int) -> None:
    if rc != QGPU_OK:
        raise QgpuError(rc, load().qgpu_last_error().decode(errors="replace"))


def config(**kw) -> Config:
    cfg = Config()
    _check(load().qgpu_config_init(ctypes.byref(cfg)))
    for k, v in kw.items():
        if k == "nccl_unique_id" and v is not None and not isinstance(v, int):
            buf = ctypes.create_string_buffer(bytes(v), 128)
            cfg._nccl_id_buf = buf  # keep alive
            v = ctypes.addressof(buf)
        setattr(cfg, k, v)
    return cfg


class Circuit:
    """A parsed OpenQASM-2 circuit (qgpu_circuit_from_qasm)."""

    def __init__(self, qasm_text: str):
        lib = load()
        self._h = ctypes.c_void_p()
        data = qasm_text.encode()
        _check(lib.qgpu_circuit_from_qasm(data, len(data), ctypes.byref(self._h)))

    @property
    def handle(self):
        return self._h

    def info(self):
        n, g = ctypes.c_int(), ctypes.c_uint64()
        _check(load().qgpu_circuit_info(self._h, ctypes.byref(n), ctypes.byref(g)))
        return n.value, g.value

    def reorder(self, mode: int) -> np.ndarray:
        _, ng = self.info()
        out = np.zeros(max(ng, 1), dtype=np.uint64)
        cnt = ctypes.c_uint64()
        _check(load().qgpu_circuit_reorder(self._h, mode, out.ctypes.data, ng, ctypes.byref(cnt)))
        return out[:cnt.value].astype(np.int64)

    def plan(self, n: int, world_size: int = 1, reorder: int = 2, fuse_bits: int = 12) -> np.ndarray:
        cnt = ctypes.c_uint64()
        _check(load().qgpu_circuit_plan(self._h, n, world_size, reorder, fuse_bits, None, 0,
                                        ctypes.byref(cnt)))
        info = np.zeros((max(cnt.value, 1), 8), dtype=np.int64)
        _check(load().qgpu_circuit_plan(self._h, n, world_size, reorder, fuse_bits,
                                        info.ctypes.data, cnt.value, ctypes.byref(cnt)))
        return info[:cnt.value]

    def plan_text(self, n: int, world_size: int = 1, reorder: int = 2, fuse_bits: int = 12) -> str:
        ln = ctypes.c_size_t()
        _check(load().qgpu_circuit_plan_text(self._h, n, world_size, reorder, fuse_bits, None, 0,
                                             ctypes.byref(ln)))
        buf = ctypes.create_string_buffer(ln.value + 1)
        _check(load().qgpu_circuit_plan_text(self._h, n, world_size, reorder, fuse_bits, buf,
                                             ln.value + 1, ctypes.byref(ln)))
        return buf.value.decode()

    def jit_check(self, n: int, reorder: int = 2, fuse_bits: int = 12) -> int:
        """Compile the NVRTC-specialised kernel of every fused pass (no GPU needed)."""
        k = ctypes.c_int()
        _check(load().qgpu_circuit_jit_check(self._h, n, reorder, fuse_bits, ctypes.byref(k)))
        return k.value

    def close(self):
        if self._h:
            load().qgpu_circuit_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class State:
    """An n-qubit state vector on one GPU (or one shard of it), starting in |0...0>."""

    def __init__(self, n: int, cfg: Optional[Config] = None, **kw):
        lib = load()
        if kw.get("nccl_unique_id") is not None and "QGPU_NCCL_LIB" not in os.environ and _nccl_lib_path():
            os.environ["QGPU_NCCL_LIB"] = _nccl_lib_path()
        self.cfg = cfg if cfg is not None else config(**kw)
        self._h = ctypes.c_void_p()
        _check(lib.qgpu_state_create(n, ctypes.byref(self.cfg), ctypes.byref(self._h)))
        self.n = n

    @property
    def handle(self):
        return self._h

    def close(self):
        if self._h:
            load().qgpu_state_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def reset(self):
        _check(load().qgpu_state_reset(self._h))

    def synchronize(self):
        _check(load().qgpu_synchronize(self._h))

    def info(self):
        n, nl, p = ctypes.c_int(), ctypes.c_int(), ctypes.c_void_p()
        _check(load().qgpu_state_info(self._h, ctypes.byref(n), ctypes.byref(nl), ctypes.byref(p)))
        return n.value, nl.value, p.value

    def set_amplitudes(self, psi: np.ndarray):
        psi = np.ascontiguousarray(psi, dtype=np.complex128)
        assert psi.size == 1 << self.n
        _check(load().qgpu_set_amplitudes(self._h, psi.ctypes.data))

    def apply_gate(self, U, targets: Sequence[int], controls: Sequence[int] = ()):
        U = np.ascontiguousarray(U, dtype=np.complex128)
        t = np.ascontiguousarray(targets, dtype=np.int32)
        c = np.ascontiguousarray(controls if len(controls) else [0], dtype=np.int32)
        assert U.shape == (1 << len(t), 1 << len(t))
        _check(load().qgpu_apply_gate(self._h, U.ctypes.data, len(t), t.ctypes.data, len(controls),
                                      c.ctypes.data if len(controls) else None))

    def apply_circuit(self, circ: Circuit):
        _check(load().qgpu_apply_circuit(self._h, circ.handle))

    def apply_circuit_probabilities(self, circ: Circuit, qubits: Sequence[int]) -> np.ndarray:
        """Apply `circ` and return the marginal probabilities of `qubits` at its end (fused into
        the last pass when possible; qgpu_apply_circuit_probabilities)."""
        q = np.ascontiguousarray(qubits if len(qubits) else [0], dtype=np.int32)
        out = np.empty(1 << len(qubits), dtype=np.float64)
        _check(load().qgpu_apply_circuit_probabilities(self._h, circ.handle, len(qubits), q.ctypes.data,
                                                       out.ctypes.data))
        return out

    def amplitudes(self, start: int = 0, count: Optional[int] = None) -> np.ndarray:
        if count is None:
            count = (1 << self.n) - start
        out = np.empty(count, dtype=np.complex128)
        _check(load().qgpu_get_amplitudes(self._h, start, count, out.ctypes.data))
        return out

    def amplitudes_device(self, start: int, count: int, dev_ptr: int):
        _check(load().qgpu_get_amplitudes_device(self._h, start, count, dev_ptr))

    def probabilities(self, qubits: Sequence[int]) -> np.ndarray:
        q = np.ascontiguousarray(qubits if len(qubits) else [0], dtype=np.int32)
        out = np.empty(1 << len(qubits), dtype=np.float64)
        _check(load().qgpu_probabilities(self._h, len(qubits), q.ctypes.data, out.ctypes.data))
        return out

    def involvement(self) -> int:
        v = ctypes.c_uint64()
        _check(load().qgpu_get_involvement(self._h, ctypes.byref(v)))
        return v.value

    def chunk_bitmap(self, chunk_bits: int) -> np.ndarray:
        nch = 1 << (self.n - chunk_bits)
        words = np.zeros((nch + 63) // 64, dtype=np.uint64)
        _check(load().qgpu_get_chunk_bitmap(self._h, chunk_bits, words.ctypes.data, words.size))
        bits = np.unpackbits(words.view(np.uint8), bitorder="little")[:nch]
        return bits.astype(np.uint8)

    def schedule(self):
        cnt = ctypes.c_uint64()
        _check(load().qgpu_get_schedule(self._h, None, None, 0, ctypes.byref(cnt)))
        o = np.zeros(max(cnt.value, 1), dtype=np.uint64)
        iv = np.zeros(max(cnt.value, 1), dtype=np.uint64)
        _check(load().qgpu_get_schedule(self._h, o.ctypes.data, iv.ctypes.data, cnt.value,
                                        ctypes.byref(cnt)))
        return o[:cnt.value].astype(np.int64), iv[:cnt.value]

    def qubit_map(self) -> np.ndarray:
        pos = np.zeros(self.n, dtype=np.int32)
        _check(load().qgpu_get_qubit_map(self._h, pos.ctypes.data))
        return pos

    def stats(self) -> dict:
        s = Stats()
        _check(load().qgpu_get_stats(self._h, ctypes.byref(s)))
        return s.as_dict()

    def reset_stats(self):
        _check(load().qgpu_reset_stats(self._h))

    def set_timing(self, mode: int):
        _check(load().qgpu_set_timing(self._h, mode))

    def pass_profile(self) -> list:
        """Per-pass records (cfg timing=2) since the last call / reset (qgpu_get_pass_profile)."""
        cnt = ctypes.c_uint64()
        _check(load().qgpu_get_pass_profile(self._h, None, 0, ctypes.byref(cnt)))
        arr = (PassProfile * max(cnt.value, 1))()
        _check(load().qgpu_get_pass_profile(self._h, arr, cnt.value, ctypes.byref(cnt)))
        return [arr[i].as_dict() for i in range(cnt.value)]


def _nccl_lib_path():
    try:
        import nvidia.nccl
        for d in nvidia.nccl.__path__:
            p = os.path.join(d, "lib", "libnccl.so.2")
            if os.path.exists(p):
                return p
    except Exception:
        pass
    return None


def nccl_unique_id() -> bytes:
    """A fresh ncclUniqueId (128 bytes) to broadcast from rank 0 (torch.distributed)."""
    if "QGPU_NCCL_LIB" not in os.environ and _nccl_lib_path():
        os.environ["QGPU_NCCL_LIB"] = _nccl_lib_path()
    buf = ctypes.create_string_buffer(128)
    _check(load().qgpu_nccl_unique_id(buf, 128))
    return buf.raw


def gfc_max_bytes(n: int, seg_len: int) -> int:
    """Largest compressed size of n doubles (qgpu_gfc_max_bytes)."""
    out = ctypes.c_uint64()
    _check(load().qgpu_gfc_max_bytes(n, seg_len, ctypes.byref(out)))
    return out.value


def gfc_compress(d_in: int, n: int, seg_len: int, d_out: int, out_cap: int, d_offsets: int,
                 stream: int = 0) -> int:
    """GFC-compress n doubles at device address d_in into d_out / d_offsets (device
    addresses); returns the compressed size in bytes (qgpu_gfc_compress, synchronising)."""
    out = ctypes.c_uint64()
    _check(load().qgpu_gfc_compress(d_in, n, seg_len, d_out, out_cap, d_offsets, ctypes.byref(out),
                                    stream or None))
    return out.value


def gfc_decompress(d_in: int, d_offsets: int, n: int, seg_len: int, d_out: int, stream: int = 0) -> None:
    """Inverse of gfc_compress (device addresses; asynchronous on `stream`)."""
    _check(load().qgpu_gfc_decompress(d_in, d_offsets, n, seg_len, d_out, stream or None))


def measure_fp64_peak(device: int = 0) -> float:
    """Thread-level DFMA per second of `device` (qgpu_measure_fp64_peak)."""
    out = ctypes.c_double()
    _check(load().qgpu_measure_fp64_peak(device, ctypes.byref(out)))
    return out.value


def version() -> str:
    return load().qgpu_version().decode()
