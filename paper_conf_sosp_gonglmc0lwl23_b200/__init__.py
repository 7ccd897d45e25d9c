"""B200-native gSampler ECSF sampling hot path (GraphSAGE, KGCN, PASS-style,
ShaDow, LADIES/FastGCN, DeepWalk/Node2Vec) behind the C ABI in include/gs.h.

The CUDA library is loaded lazily by ``paper_conf_sosp_gonglmc0lwl23_b200.gs``;
there is no CPU fallback.
"""
__all__ = ["gs", "build", "dist"]
