"""B200-native GROPHECY++ projection engine (Boyer, Meng, Kumaran, IPDPS 2013).

The product path is the CUDA library libgrophecy.so (C ABI in
include/grophecy.h); ``grophecy`` is its thin ctypes binding and ``dist``
the torch.distributed glue for the multi-GPU min-loc.  Importing ``grophecy``
fails loudly if the library has not been built — there is no CPU fallback.
"""
__all__ = ["grophecy", "dist", "build"]
