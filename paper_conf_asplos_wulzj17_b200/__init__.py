"""FLEP on B200: preemptable persistent-CTA kernels + the FLEP runtime, behind a C ABI.

The product is libflep.so (include/flep.h); this package is its ctypes binding (`flep`) and
build script (`build`). See DESIGN.md.
"""
import os as _os

# More hardware work queues than CUDA's default 8, so the runtime's control stream and the
# execution streams do not falsely serialise behind each other (must precede CUDA init).
_os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

from . import flep  # noqa: F401,E402
from .flep import Runtime, PolicyEngine  # noqa: F401,E402
