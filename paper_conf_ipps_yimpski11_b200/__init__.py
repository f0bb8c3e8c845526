"""HAUBERK hot path for B200 (sm_100a): SDC-detector-instrumented CP / MRI-Q / TPACF kernels,
value-range profiler, seeded single-bit injector and replica-mode coverage campaign.

The compute path is libhauberk.so (csrc/, C ABI in include/hauberk.h); `hauberk` is its ctypes
binding and `parallel` shards campaigns across GPUs with torch.distributed (NCCL)."""
from . import hauberk  # noqa: F401

__all__ = ["hauberk"]
