"""Real-UM runtime: argument
marshalling over libdeepum_um.so, whose C-ABI is include/deepum_um.h.

    um = UmRuntime(n_blocks, device=0)      # managed arena of 2 MiB UM blocks
    um.intercept(True, faults=True)          # CUPTI: exec-ID hashes of every launch (+ UM fault records)
    ...                                      # kernels run over the arena
    hashes, offs, faults = um.take()         # dum_record_faults layout
    um.prefetch(blocks, to_device=True)      # cudaMemPrefetchAsync per run of blocks
"""
from __future__ import annotations

import ctypes
import os
from typing import Tuple

import numpy as np
import torch

from . import binding as B

_HERE = os.path.dirname(os.path.abspath(__file__))
_PATH = os.path.join(_HERE, "libdeepum_um.so")
_LIB = None


def load_um_library() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(_PATH):
        raise ImportError("libdeepum_um.so is not built (python -m paper_conf_asplos_jungkl23_b200.build)")
    L = ctypes.CDLL(_PATH)
    P, U32, U64, I = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    for name, res, args in [("dum_um_create", P, [U32, I]), ("dum_um_destroy", None, [P]),
                            ("dum_um_base", P, [P]), ("dum_um_last_error", ctypes.c_char_p, [P]),
                            ("dum_um_intercept", I, [P, I, I]), ("dum_um_fault_source", I, [P, P, U32]),
                            ("dum_um_add_faults", I, [P, P, U32]),
                            ("dum_um_take", I, [P, P, P, P, U32, U64, P, P, P]),
                            ("dum_um_prefetch", I, [P, P, U32, I, P]), ("dum_um_touch", I, [P, P, U32, P])]:
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


class UmRuntime:
    def __init__(self, n_blocks: int, device: int = 0):
        self.lib = load_um_library()
        self.n_blocks = n_blocks
        self.device = torch.device("cuda", device)
        self._h = self.lib.dum_um_create(n_blocks, device)
        if not self._h:
            raise RuntimeError("dum_um_create failed (cudaMallocManaged of %d x 2 MiB)" % n_blocks)

    def close(self):
        if getattr(self, "_h", None):
            self.lib.dum_um_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def _ck(self, rc: int, what: str) -> None:
        if rc != 0:
            raise B.EngineError(rc, "%s: %s" % (what, self.lib.dum_um_last_error(self._h).decode()))

    def _stream(self):
        return ctypes.c_void_p(torch.cuda.current_stream(self.device).cuda_stream)

    @property
    def base(self) -> int:
        return int(self.lib.dum_um_base(self._h))

    def intercept(self, enable: bool = True, faults: bool = True) -> None:
        self._ck(self.lib.dum_um_intercept(self._h, 1 if enable else 0, 1 if faults else 0), "dum_um_intercept")

    def fault_source(self) -> Tuple[bool, str]:
        buf = ctypes.create_string_buffer(256)
        r = self.lib.dum_um_fault_source(self._h, buf, 256)
        return r == 1, buf.value.decode()

    def add_faults(self, blocks) -> None:
        a = np.ascontiguousarray(blocks, dtype=np.uint32)
        self._ck(self.lib.dum_um_add_faults(self._h, a.ctypes.data, a.size), "dum_um_add_faults")

    def take(self, launch_cap: int = 1 << 16, fault_cap: int = 1 << 22):
        """(hashes u64[n], offsets u64[n+1], faults u32[m]) of the launches since the last take."""
        h = np.zeros(launch_cap, np.uint64)
        o = np.zeros(launch_cap + 1, np.uint64)
        f = np.zeros(fault_cap, np.uint32)
        nl, nf = ctypes.c_uint32(0), ctypes.c_uint64(0)
        need = np.zeros(2, np.uint64)
        self._ck(self.lib.dum_um_take(self._h, h.ctypes.data, o.ctypes.data, f.ctypes.data, launch_cap, fault_cap,
                                      ctypes.byref(nl), ctypes.byref(nf), need.ctypes.data), "dum_um_take")
        n, m = nl.value, nf.value
        return h[:n].copy(), o[:n + 1].copy(), f[:m].copy()

    def prefetch(self, blocks, to_device: bool = True) -> None:
        a = np.ascontiguousarray(blocks, dtype=np.uint32)
        self._ck(self.lib.dum_um_prefetch(self._h, a.ctypes.data, a.size, 1 if to_device else 0, self._stream()),
                 "dum_um_prefetch")

    def touch(self, blocks_dev: torch.Tensor) -> None:
        assert blocks_dev.is_cuda and blocks_dev.dtype == torch.int32
        self._ck(self.lib.dum_um_touch(self._h, ctypes.c_void_p(blocks_dev.data_ptr()), blocks_dev.numel(),
                                       self._stream()), "dum_um_touch")
