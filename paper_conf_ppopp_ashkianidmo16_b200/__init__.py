"""B200-native stable multisplit (Ashkiani, Davidson, Meyer, Owens, PPoPP'16).

C ABI: include/ms.h (libms.so, built in-tree by build.py); this package is its
thin Python binding.  See DESIGN.md.
"""
from .api import BucketSpec, Plan, multisplit  # noqa: F401
from ._abi import MultisplitError  # noqa: F401
