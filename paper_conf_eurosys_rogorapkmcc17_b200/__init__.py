"""B200-native TagMatch: GPU subset matching of Bloom-filter tag-set signatures.

The product is the C-ABI library libtagmatch.so (include/tagmatch.h); this
package holds its CUDA/C++ sources (csrc/), the in-tree build (_build.py) and a
thin ctypes binding (tagmatch.py).  Every step of the matching path runs in the
library's sm_100a kernels; there is no CPU fallback.
"""
from .tagmatch import (Database, HostTagSets, TagMatchError, abi_version, device_tagsets, encode, load,  # noqa: F401
                       TM_DEFAULT_MAX_PARTITION, TM_NO_PARTITIONING, TM_AUTO_MAX_PARTITION, EXPORTS, LIB_PATH)
