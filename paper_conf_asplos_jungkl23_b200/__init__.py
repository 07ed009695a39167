"""B200-native DeepUM correlation-prefetch and tensor-migration engine.

Thin Python binding (argument marshalling only) over libdeepum_b200.so, whose
C-ABI is include/deepum_b200.h.  Every step of the hot path runs in that
library's CUDA kernels; PyTorch is used only for device memory and streams.
There is no CPU fallback: if the library is missing this package refuses to
import.
"""
from .binding import (  # noqa: F401
    DUM_NONE, NONE, Engine, EngineError, load_library, library_path,
    DUMP_EXEC, DUMP_CORR, DUMP_BLK, DUMP_WALK, DUMP_RES, DUMP_HIST,
    H2D, D2H, INVALIDATE, D2D,
)
