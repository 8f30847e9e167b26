"""B200-native Local Field Dynamics (LFD) step of DC-MESH (Razakh et al., IPDPS-W 2024).

The product is the C-ABI CUDA library ``liblfd.so`` (include/lfd.h, sources in csrc/); ``lfd`` is the
thin ctypes binding with the same entry-point names.
"""
from . import lfd  # noqa: F401
from .lfd import Context, LFDError  # noqa: F401
