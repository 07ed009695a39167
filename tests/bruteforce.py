"""Independent brute-force statistics used to PIN the oracle (not a second copy
of it).  Each function computes a quantity that the paper's definitions fix
directly, without the oracle's table machinery:

  dedupe_first         PAPER.md L124 step (2) "removes the duplicate addresses
                       and groups them according to their UM blocks" (D2)
  dense_exec_ids       PAPER.md L136: same hash -> same ID, else a new ID
  successor_lists      PAPER.md L168 "NumSucc entries are MRU ordered": with no
                       row replacement a row holds the S most recent distinct
                       successors of its block
  lru_tags             a set with R=1 rows is a textbook A-entry LRU cache
  next_exec            PAPER.md L208: the record predicts the kernel that
                       followed the 3-kernel history last time
  select_victims       PAPER.md L238-L241: least recently migrated first, skip
                       blocks expected in the window; L285 split by inactivity
"""
from __future__ import annotations

from typing import Dict, Iterable, List, Optional, Sequence, Tuple

NONE = 0xFFFFFFFF


def dedupe_first(seq: Iterable[int]) -> List[int]:
    seen = set()
    out = []
    for x in seq:
        if x not in seen:
            seen.add(x)
            out.append(x)
    return out


def dense_exec_ids(hashes: Sequence[int]) -> List[int]:
    m: Dict[int, int] = {}
    return [m.setdefault(int(h), len(m)) for h in hashes]


def successor_lists(launch_lists: Sequence[Sequence[int]], S: int) -> Dict[int, List[int]]:
    """For one exec ID: launch_lists are its (deduplicated) fault lists in
    order.  Returns {block: most recent distinct successors, newest first}."""
    pairs: List[Tuple[int, int]] = []
    blocks = set()
    for L in launch_lists:
        blocks.update(L)
        for i in range(1, len(L)):
            pairs.append((L[i - 1], L[i]))
    out: Dict[int, List[int]] = {b: [] for b in blocks}
    for p, s in reversed(pairs):
        if s == p:
            continue
        lst = out[p]
        if s not in lst and len(lst) < S:
            lst.append(s)
    return out


def lru_tags(touches: Sequence[int], A: int) -> List[int]:
    cache: List[int] = []
    for b in touches:
        if b in cache:
            cache.remove(b)
        cache.insert(0, b)
        del cache[A:]
    return cache


def next_exec(exec_seq: Sequence[int], e: int, h: Tuple[int, int, int]) -> int:
    """Successor of the last occurrence of the 4-gram (h1,h2,h3,e) followed by
    some kernel, with NONE padding before the first launch."""
    padded = [NONE, NONE, NONE] + list(exec_seq)
    ans = NONE
    for k in range(3, len(padded) - 1):
        if tuple(padded[k - 3:k]) == tuple(h) and padded[k] == e:
            ans = padded[k + 1]
    return ans


def select_victims(lrm: Sequence[int], n_free: int, window: Sequence[int], anchor: int,
                   resident: set, inactive: set) -> Tuple[List[int], List[int]]:
    wset = set(window)
    if anchor != NONE:
        wset.add(anchor)
    nonres = sum(1 for b in window if b not in resident)
    need = max(0, nonres - n_free)
    victims = [b for b in lrm if b not in wset][:need]
    return [b for b in victims if b not in inactive], [b for b in victims if b in inactive]
