"""paper_conf_icpp_bastemuzas17_b200 — B200-native tiled, stream-pipelined
fp64 heat stencil (Bastem et al., ICPP 2017).

The product is libtiles.so (C ABI in include/tiles.h; CUDA kernels for
sm_100a in csrc/). `tiles` is its thin ctypes binding.
"""
from . import tiles  # noqa: F401  (raises ImportError if libtiles.so is missing)
from .tiles import Domain, heat7, sincos, nccl_unique_id, TileError  # noqa: F401

__all__ = ["tiles", "Domain", "heat7", "sincos", "nccl_unique_id", "TileError"]
