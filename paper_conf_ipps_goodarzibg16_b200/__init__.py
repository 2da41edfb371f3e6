"""B200-native GP-metis coarsening path (Goodarzi, Burtscher, Goswami, IPDPS-W 2016).

The product is libgpcoarsen.so (sm_100a CUDA kernels behind the C ABI of include/gp.h);
``paper_conf_ipps_goodarzibg16_b200.gp`` is its ctypes binding.  Import ``gp`` explicitly:
it raises if the library has not been built (there is no CPU fallback).
"""
__all__ = ["gp"]
