"""B200-native TileSpMSpV / TileBFS (Ji et al., ICPP '22).

The compute path is libtsmv.so (hand-written sm_100a CUDA, C ABI in
include/tsmv.h); `tsmv` is its ctypes binding and `dist` the row-block
multi-GPU driver on top of torch.distributed.  Importing `tsmv` fails loudly if
the library has not been built: there is no CPU fallback.
"""
__all__ = ["tsmv", "dist", "build"]
