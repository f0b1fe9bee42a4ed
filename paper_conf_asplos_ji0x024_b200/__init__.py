"""B200-native multi-scalar multiplication (Pippenger buckets, XYZZ) — DistMSM's hot path.

The product is the C-ABI library `libmsm.so` (include/msm.h, sources in csrc/); this
package is its thin ctypes binding (msm.py).  PyTorch is used by callers only for device
memory, streams and torch.distributed; it is not needed to import this package.
"""
from .msm import (CURVE_IDS, Context, MSMError, debug_digits, debug_ec, debug_field, device_count,  # noqa: F401
                  field_words, finalize, gen_points, lib, partial_words, scalar_words)
