"""B200-native nested-method correlated subquery engine (NestGPU hot path).

The engine is libnestgpu.so (include/nestgpu.h, hand-written CUDA for
sm_100a); :class:`Engine` is its argument-marshalling binding.  See DESIGN.md.
"""
from .binding import (Engine, NestGPUError, load_library, LIB_PATH, SYMBOLS,  # noqa: F401
                      DT, CMP, AGG, STAGES, STRATEGIES, cost_estimate)
