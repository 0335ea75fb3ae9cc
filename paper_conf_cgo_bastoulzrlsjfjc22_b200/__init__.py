"""B200-native fused memory-bound operators (Bastoul et al., CGO'22 hot path).

Public API: ``FusedOp(desc, **opts)`` plans a fused operator (validation,
Algorithm-2 vectorisation planner, kernel generation + NVRTC compilation for
sm_100a, all inside libfop.so) and ``FusedOp.run(tensors)`` launches it on the
current CUDA stream.  ``dist`` shards fused operators over GPUs.

The binding (and libfop.so) is loaded on first use of an exported name, so
``python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build`` works before the
library exists.
"""
_EXPORTS = ("FusedOp", "FopError", "abi_version", "marshal", "default_opts", "ABI_SYMBOLS", "LIB_PATH",
            "run_host_many", "run_many", "PeerGroup", "peer_alloc", "peer_free", "peer_open", "peer_close")

__all__ = list(_EXPORTS)


def __getattr__(name):
    if name in _EXPORTS:
        from . import fop
        return getattr(fop, name)
    raise AttributeError(name)
