"""B200-native CSWAP hot path: compressed tensor swapping (ZVC/RLE/CSR/LZ4) on sm_100a.

The product is the C-ABI library ``libcswap.so`` (include/cswap.h); ``cswap`` is its thin
ctypes binding.  Build with ``python -m paper_conf_cluster_chenhzchysc21_b200.build``.
"""
