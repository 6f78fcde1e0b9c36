"""B200-native HIOS executor: batch-1 DAG-CNN inference under an HIOS-LP
schedule (Kundu & Shu, CLUSTER 2023).  The product is libhios.so (C-ABI,
include/hios.h); ``hios`` is its thin ctypes binding."""
from . import hios  # noqa: F401

__all__ = ["hios"]
