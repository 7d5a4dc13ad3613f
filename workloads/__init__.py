"""Seeded synthetic workload generators (QASM text). Shared by oracle and product; holds no
arithmetic of the method (see circuits.py)."""
from .circuits import *  # noqa: F401,F403
