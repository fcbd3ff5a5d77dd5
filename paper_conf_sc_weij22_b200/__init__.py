"""B200-native STMatch counting hot path (Wei & Jiang, SC'22).

The product is ``libstm.so`` (include/stm.h): a host pattern compiler and one
persistent sm_100a CUDA kernel.  ``stm`` is the ctypes binding (marshalling
only); ``dist`` is the 1..8 GPU layer over torch.distributed.
"""
__all__ = ["stm", "dist", "build"]
