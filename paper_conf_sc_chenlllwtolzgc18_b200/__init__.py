"""B200-native two-dimensional weighted-checksum ABFT (Chen et al., SC'18).

The product is libabft_b200.so (sm_100a CUDA + cuBLAS/cuSOLVER behind the C
ABI of include/abft.h); `abft` is its thin ctypes binding.  Import
`paper_conf_sc_chenlllwtolzgc18_b200.abft` to load the library."""
__all__ = ["abft"]
