"""B200-native (sm_100a) q4-KV decode-attention hot path of LM-Offload.

The product is the C-ABI library ``liblmo.so`` (include/lmo.h); ``lmo`` is a
thin ctypes binding over it.  Importing this package does not load CUDA code;
``from paper_conf_ipps_wurypgll25_b200 import lmo`` does, and fails loudly if
the library is missing.
"""
__all__ = ["configs", "inputs"]
