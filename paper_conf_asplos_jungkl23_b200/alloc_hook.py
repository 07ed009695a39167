"""PyTorch allocator hook for inactive-block tracking (
PAPER.md L283-L285): argument marshalling over libdeepum_hook.so, whose C-ABI
is include/deepum_hook.h.

    hook = AllocHook(max_blocks=engine_W, device=0)
    hook.attach()            # existing segments from torch.cuda.memory_snapshot(), then the tracker
    ...                      # training step: allocations / frees are tracked
    hook.flush(engine)       # queued UM blocks -> dum_mark_inactive (active / inactive)
"""
from __future__ import annotations

import ctypes
import os
from typing import Tuple

import numpy as np
import torch

from . import binding as B

_HERE = os.path.dirname(os.path.abspath(__file__))
_PATH = os.path.join(_HERE, "libdeepum_hook.so")
_LIB = None

ALLOC, FREE_REQUESTED, FREE_COMPLETED, SEGMENT_ALLOC, SEGMENT_FREE, SEGMENT_MAP, SEGMENT_UNMAP = range(7)


def load_hook_library() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(_PATH):
        raise ImportError("libdeepum_hook.so is not built (python -m paper_conf_asplos_jungkl23_b200.build)")
    B.load_library()  # libdeepum_b200.so first (the hook calls dum_mark_inactive)
    L = ctypes.CDLL(_PATH)
    P, U32, U64, I = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    for name, res, args in [("dum_hook_create", P, [U32, I]), ("dum_hook_destroy", None, [P]),
                            ("dum_hook_attach", I, [P]), ("dum_hook_feed", I, [P, I, U64, U64]),
                            ("dum_hook_block_of", U32, [P, U64]),
                            ("dum_hook_drain", I, [P, P, P, P, P, U32]), ("dum_hook_flush", I, [P, P, P]),
                            ("dum_hook_stats", I, [P, P])]:
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


class AllocHook:
    def __init__(self, max_blocks: int, device: int = 0):
        self.lib = load_hook_library()
        self.device = device
        self._h = self.lib.dum_hook_create(max_blocks, device)
        if not self._h:
            raise ValueError("dum_hook_create: bad arguments")

    def __del__(self):
        if getattr(self, "_h", None):
            self.lib.dum_hook_destroy(self._h)
            self._h = None

    def _ck(self, rc: int, what: str) -> None:
        if rc != 0:
            raise B.EngineError(rc, what)

    def feed(self, action: int, addr: int, size: int) -> None:
        self._ck(self.lib.dum_hook_feed(self._h, action, addr, size), "dum_hook_feed")

    def feed_snapshot(self) -> None:
        """The caching allocator's current segments and live blocks (events from
        before attach()) as SEGMENT_ALLOC / ALLOC events."""
        for seg in torch.cuda.memory_snapshot():
            if seg.get("device") != self.device:
                continue
            self.feed(SEGMENT_ALLOC, int(seg["address"]), int(seg["total_size"]))
            a = int(seg["address"])
            for blk in seg.get("blocks", []):
                if blk.get("state") in ("active_allocated", "active_pending_free"):
                    self.feed(ALLOC, int(blk.get("address", a)), int(blk["size"]))
                a += int(blk["size"])

    def attach(self, snapshot: bool = True) -> None:
        if snapshot:
            self.feed_snapshot()
        self._ck(self.lib.dum_hook_attach(self._h), "dum_hook_attach")

    def block_of(self, addr: int) -> int:
        return int(self.lib.dum_hook_block_of(self._h, addr))

    def drain(self, cap: int = 1 << 20) -> Tuple[np.ndarray, np.ndarray]:
        """(blocks now inactive, blocks now active), ascending."""
        ina = np.zeros(cap, dtype=np.uint32)
        act = np.zeros(cap, dtype=np.uint32)
        ni, na = ctypes.c_uint32(0), ctypes.c_uint32(0)
        rc = self.lib.dum_hook_drain(self._h, ina.ctypes.data, ctypes.byref(ni), act.ctypes.data, ctypes.byref(na),
                                     cap)
        if rc < 0:
            raise B.EngineError(-2, "dum_hook_drain: more queued blocks than cap")
        return ina[: ni.value].copy(), act[: na.value].copy()

    def flush(self, engine) -> None:
        s = torch.cuda.current_stream(engine.device).cuda_stream
        self._ck(self.lib.dum_hook_flush(self._h, engine._h, ctypes.c_void_p(s)), "dum_hook_flush")

    def stats(self) -> dict:
        out = np.zeros(4, dtype=np.uint64)
        self._ck(self.lib.dum_hook_stats(self._h, out.ctypes.data), "dum_hook_stats")
        return {"events": int(out[0]), "dropped": int(out[1]), "blocks": int(out[2]), "live_bytes": int(out[3])}
