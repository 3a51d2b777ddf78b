"""B200-native zonal histogramming (Zhang & Wang, IPDPS-W 2014, dblp conf/ipps/ZhangW14).

The product is libzh.so (include/zh.h, sm_100a CUDA in csrc/); `zh` is its ctypes binding and
`dist` the tile-row sharding + NCCL reduce used for multi-GPU runs.
"""
from ._build import LIB as LIB_PATH  # noqa: F401
