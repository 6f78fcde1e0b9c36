"""Workload data shared by the oracle and the CUDA path: graph structure and
seeded random inputs/weights only (no arithmetic of the method)."""
from . import gen, graphs  # noqa: F401
