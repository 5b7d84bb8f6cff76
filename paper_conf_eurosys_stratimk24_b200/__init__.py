"""B200-native Orion (EuroSys '24) hot path: liborion (C++ scheduler + sm_100a kernels) + binding."""
from . import _lib  # noqa: F401  (raises if liborion.so is missing: no fallback)
from .runtime import Orion, make_op, op_array, kernel_launch, kernel_geometry, now_ns, f32bits  # noqa: F401
