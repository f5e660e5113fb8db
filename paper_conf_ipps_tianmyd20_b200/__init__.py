"""B200-native PCGCN hot path: partition-centric GCN aggregation with a
dual-mode (selective CSR gather / full tcgen05 tile) executor.

The product is libpcgcn.so (C ABI in include/pcgcn.h); `_lib` is its thin
ctypes binding and `gcn` the 2-layer GCN step built on it.  There is no CPU
fallback.
"""
__all__ = ["_lib", "gcn"]
