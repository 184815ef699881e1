"""npp — B200-native mapping of nested parallel patterns (Lee et al., MICRO'14).

The product is libnpp.so (include/npp.h); ``npp`` is its ctypes binding and ``dist`` the multi-GPU
driver over torch.distributed.  Import ``paper_conf_micro_leebsro14_b200.npp`` explicitly: it raises if
the library has not been built (there is no CPU fallback).
"""
