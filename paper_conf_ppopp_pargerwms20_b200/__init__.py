"""B200-native spECK: row-wise (Gustavson) CSR SpGEMM C = A·B with lightweight analysis,
global/local load balancing and hash / dense / direct accumulators (Parger et al.,
PPoPP'20), as hand-written sm_100a CUDA kernels behind a C ABI (include/speck.h).

The Python layer is argument marshalling over libspeck.so (speck.py) plus the row-block
multi-GPU partitioner (dist.py).  There is no CPU fallback.
"""
from .speck import (CSR, Handle, SpeckError, Stats, default_handle, load, spgemm, version,  # noqa: F401
                    EXPORTS, LIB_PATH, OPT)

__all__ = ["CSR", "Handle", "SpeckError", "Stats", "default_handle", "load", "spgemm", "version", "EXPORTS",
           "LIB_PATH", "OPT"]
