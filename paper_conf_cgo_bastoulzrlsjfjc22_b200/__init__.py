"""B200-native fused memory-bound operators (Bastoul et al., CGO'22 hot path).

Public API: ``FusedOp(desc, **opts)`` plans a fused operator (validation,
Algorithm-2 vectorisation planner, kernel generation + NVRTC compilation for
sm_100a, all inside libfop.so) and ``FusedOp.run(tensors)`` launches it on the
current CUDA stream.  ``dist`` shards fused operators over GPUs.
"""
from .fop import FusedOp, FopError, abi_version, marshal, default_opts, ABI_SYMBOLS, LIB_PATH

__all__ = ["FusedOp", "FopError", "abi_version", "marshal", "default_opts", "ABI_SYMBOLS", "LIB_PATH"]
