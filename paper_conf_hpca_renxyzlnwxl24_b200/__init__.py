"""B200-native DyNN-Offload hot path: pilot -> decode -> plan -> migrate (libdyo.so).

The product path is libdyo.so (include/dyo.h) — hand-written sm_100a CUDA kernels plus a C++
DMA engine; `dyo` is its thin ctypes binding. No CPU fallback exists.
"""
from .dyo import Dyo, DyoError, Trainer, lib, LIB_PATH, EXPORTS  # noqa: F401
