"""B200-native Liger hot path: interleaved tensor-parallel decoder serving.

The product is libliger.so (C ABI in include/liger.h); `liger` is its thin
ctypes binding and `engine` a small Python convenience layer over the serving
calls (liger_init / liger_load_layer / liger_submit / liger_step / liger_poll).
"""
from . import liger  # noqa: F401
