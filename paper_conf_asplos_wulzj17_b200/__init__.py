"""FLEP on B200: preemptable persistent-CTA kernels + the FLEP runtime, behind a C ABI.

The product is libflep.so (include/flep.h); this package is its ctypes binding (`flep`) and
build script (`build`). See DESIGN.md.
"""
from . import flep  # noqa: F401
from .flep import Runtime, PolicyEngine  # noqa: F401
