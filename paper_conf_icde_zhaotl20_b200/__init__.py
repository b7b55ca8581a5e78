"""B200-native SONG (Zhao, Tan, Li; ICDE 2020): batched graph ANN search.

The product is libsong.so (C ABI, include/song.h) built from csrc/ for
sm_100a; ``song`` is its ctypes binding and ``sharded`` the multi-GPU
orchestration over torch.distributed.
"""
from .song import (SongIndex, Params, SongError, merge_topk, version, lib,  # noqa: F401
                   rp_encode, build_graph, L2, IP, COSINE, HAMMING, METRICS, EXPORTED)

__all__ = ["SongIndex", "Params", "SongError", "merge_topk", "version", "lib"]
