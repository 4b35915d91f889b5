"""B200-native batched makespan evaluation and local search over op placements and schedules
(Pesto, Hafeez et al., Middleware '21).  The C ABI is include/pesto.h (libpesto.so); `pesto`
is its thin ctypes binding.  Import it explicitly: `from paper_conf_middleware_hafeezsg021_b200
import pesto` (it raises if libpesto.so has not been built -- there is no CPU fallback).
"""

__all__ = ["pesto"]
