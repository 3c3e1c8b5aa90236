"""B200-native batched LinnOS I/O-latency classifier (the accelerated hot path of LAKE,
Fingler et al., ASPLOS '23). See DESIGN.md and include/lake_linnos.h.

Submodules:
  lake     the C-ABI binding (liblake_linnos.so: CUDA kernels for sm_100a)
  inputs   seeded synthetic traces / raw records / weights (no method arithmetic)
  shard    multi-GPU placement of per-SSD models and I/O streams (host logic)
"""
from . import lake  # noqa: F401  (loads liblake_linnos.so lazily, on first call)

__all__ = ["lake"]
