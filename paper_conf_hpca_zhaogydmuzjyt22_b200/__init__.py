"""B200-native hot path of Q-GPU (Zhao et al., HPCA 2022): complex128 state-vector gate
application with zero-amplitude pruning, delayed qubit involvement and fused HBM passes.

The product is ``libqgpu.so`` (C ABI in ``include/qgpu.h``); ``qgpu`` is its thin ctypes
binding. See DESIGN.md.
"""
from .qgpu import Circuit, Config, QgpuError, State, config, load, version  # noqa: F401
