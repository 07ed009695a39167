"""Seeded synthetic fault-trace workloads (inputs only).

This module is the ONE place both sides of the parity test draw inputs from.
It holds none of DeepUM's arithmetic: no exec-ID table, no correlation table,
no walk, no pre-eviction policy.  It models the workload DeepUM observes
("the kernel execution patterns and the memory access patterns
within the kernels are fixed and repeated in the training phase of a DNN") and
the *baseline* UM driver that produces the faults (
see um_sim.c).

Configs (BASELINE.json `configs`):
  T  tiny 4-kernel loop over 256 x 2 MiB blocks, 128 frames, 10 iterations
  B  BERT-large-shaped, 24 layers, 2x oversubscription of C = 86,016 frames
  G  GPT-2-XL-shaped, 48 layers, 4x oversubscription of C = 86,016 frames
All structural choices (tensor layout, kernel access orders, jitter) are
generator design choices recorded in DESIGN.md Sec. "Input recipe".
"""
from __future__ import annotations

import ctypes
import dataclasses
import math
import os
import subprocess
from typing import List, Optional, Sequence, Tuple

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(HERE, "libumsim.so")
NONE = 0xFFFFFFFF
BLOCK_BYTES = 2 << 20           # a UM block is 4 KB x 512 = 2 MB
HBM_FRAMES_B200 = 86_016        # 168 GiB of 2 MiB frames (~180 GB HBM3e), SURVEY Sec. 8(d)
M64 = (1 << 64) - 1


# ----------------------------------------------------------------------------
# hashing / PRNG (generator-side only)
# ----------------------------------------------------------------------------
def splitmix64(x: int) -> int:
    """One splitmix64 output for state x (x is advanced by the golden gamma)."""
    z = (x + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def fnv1a64(data: bytes) -> int:
    """FNV-1a-64: the generator's stand-in for "the hash value of the kernel's
    name and arguments"."""
    h = 0xCBF29CE484222325
    for c in data:
        h ^= c
        h = (h * 0x100000001B3) & M64
    return h


def block_fill_word(seed: int, block: int, word: int) -> int:
    """Content of 8-byte word `word` of host block `block` (SURVEY Sec. 8c a9
    checksum pin): splitmix64(seed ^ (block << 20 | word))."""
    return splitmix64((seed ^ ((block << 20) | word)) & M64)


# ----------------------------------------------------------------------------
# native FIFO (naive-UM) simulator
# ----------------------------------------------------------------------------
def _build_so() -> None:
    src = os.path.join(HERE, "um_sim.c")
    tmp = _SO + ".tmp%d" % os.getpid()
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, src])
    os.replace(tmp, _SO)


def _lib() -> ctypes.CDLL:
    src = os.path.join(HERE, "um_sim.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        _build_so()
    lib = ctypes.CDLL(_SO)
    f = lib.um_fifo_sim
    f.restype = ctypes.c_int64
    P = ctypes.c_void_p
    f.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, P, P,
                  ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint32,
                  P, P, ctypes.c_uint64, P, P]
    return lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def simulate_naive_um(W: int, C: int, access_off: np.ndarray, access_blk: np.ndarray,
                      n_iter: int, dup_seed: int = 0, dup_ppm: int = 0):
    """Fault trace of n_iter repetitions of one iteration's access stream under
    naive UM with least-recently-migrated eviction."""
    lib = _lib()
    K = len(access_off) - 1
    access_off = np.ascontiguousarray(access_off, dtype=np.uint64)
    access_blk = np.ascontiguousarray(access_blk, dtype=np.uint32)
    n = lib.um_fifo_sim(W, C, K, _ptr(access_off), _ptr(access_blk), n_iter,
                        dup_seed, dup_ppm, None, None, 0, None, None)
    if n < 0:
        raise ValueError("um_fifo_sim: bad input")
    fault_off = np.zeros(n_iter * K + 1, dtype=np.uint64)
    fault_blk = np.zeros(max(n, 1), dtype=np.uint32)
    snap_blk = np.zeros(n_iter * C, dtype=np.uint32)
    snap_cnt = np.zeros(n_iter, dtype=np.uint32)
    n2 = lib.um_fifo_sim(W, C, K, _ptr(access_off), _ptr(access_blk), n_iter,
                         dup_seed, dup_ppm, _ptr(fault_off), _ptr(fault_blk), n,
                         _ptr(snap_blk), _ptr(snap_cnt))
    assert n2 == n
    return fault_off, fault_blk[:n], snap_blk.reshape(n_iter, C), snap_cnt


# ----------------------------------------------------------------------------
# Trace container
# ----------------------------------------------------------------------------
@dataclasses.dataclass
class Trace:
    name: str
    W: int                      # block-id space (max_blocks)
    C: int                      # HBM frames
    K: int                      # launches per iteration
    n_iter: int
    launch_hash: np.ndarray     # u64 [n_iter*K]
    launch_off: np.ndarray      # u64 [n_iter*K+1] into fault_block
    fault_block: np.ndarray     # u32 [F] raw fault records (block ids)
    snap_blk: np.ndarray        # u32 [n_iter, C] resident blocks at iteration start (oldest first)
    snap_cnt: np.ndarray        # u32 [n_iter]
    inactive_blocks: np.ndarray # u32 blocks of tensors dead at an iteration boundary
    access_off: np.ndarray      # u64 [K+1]  one iteration's access stream
    access_blk: np.ndarray      # u32
    kernel_names: List[str]
    seed: int

    @property
    def n_launch(self) -> int:
        return self.n_iter * self.K

    @property
    def n_fault(self) -> int:
        return int(self.launch_off[-1])

    def iteration(self, i: int) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
        """(hash, off rebased to 0, faults) for trace iteration i."""
        return self.launches(i * self.K, (i + 1) * self.K)

    def launches(self, k0: int, k1: int) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
        h = self.launch_hash[k0:k1]
        off = self.launch_off[k0:k1 + 1]
        f = self.fault_block[int(off[0]):int(off[-1])]
        return h.copy(), (off - off[0]).astype(np.uint64), f.copy()

    def faults_in_iteration(self, i: int) -> int:
        return int(self.launch_off[(i + 1) * self.K] - self.launch_off[i * self.K])


def _jitter_hashes(base: np.ndarray, K: int, n_iter: int, seed: int, frac: float) -> np.ndarray:
    """Allocator address drift: in iteration i >= 1,
    ceil(frac*K) launch positions drawn with splitmix64(seed ^ i) get the
    fresh hash splitmix64(seed ^ i<<32 ^ pos); their block lists are unchanged."""
    out = np.tile(base.astype(np.uint64), n_iter)
    if frac <= 0:
        return out
    n_j = int(math.ceil(frac * K))
    for i in range(1, n_iter):
        st = (seed ^ i) & M64
        chosen = []
        seen = set()
        while len(chosen) < min(n_j, K):
            r = splitmix64(st)
            st = (st + 1) & M64
            p = r % K
            if p in seen:
                continue
            seen.add(p)
            chosen.append(p)
        for p in chosen:
            out[i * K + p] = np.uint64(splitmix64((seed ^ (i << 32) ^ p) & M64))
    return out


# ----------------------------------------------------------------------------
# Config T
# ----------------------------------------------------------------------------
def make_T(n_iter: int = 10, seed: int = 1, dup_ppm: int = 0) -> Trace:
    """4 tensors X_0..X_3 of 64 blocks each (X_i = blocks [64i, 64i+64)).
    Kernel i accesses all of X_i ascending, then X_{(i+1) mod 4}[0:16]."""
    W, C, K = 256, 128, 4
    offs = [0]
    blks: List[int] = []
    names = []
    for i in range(K):
        acc = list(range(64 * i, 64 * i + 64)) + list(range(64 * ((i + 1) % 4), 64 * ((i + 1) % 4) + 16))
        blks += acc
        offs.append(len(blks))
        names.append("T:k%d" % i)
    access_off = np.array(offs, dtype=np.uint64)
    access_blk = np.array(blks, dtype=np.uint32)
    base = np.array([fnv1a64(n.encode()) for n in names], dtype=np.uint64)
    fo, fb, sb, sc = simulate_naive_um(W, C, access_off, access_blk, n_iter, seed, dup_ppm)
    return Trace("T", W, C, K, n_iter, _jitter_hashes(base, K, n_iter, seed, 0.0), fo, fb, sb, sc,
                 np.zeros(0, dtype=np.uint32), access_off, access_blk, names, seed)


# ----------------------------------------------------------------------------
# Configs B and G: transformer-training-shaped traces (SURVEY Sec. 8d template)
# ----------------------------------------------------------------------------
@dataclasses.dataclass
class TransformerShape:
    name: str
    layers: int
    hidden: int
    heads: int
    seq: int
    vocab: int
    oversub: int
    adam_chunks: int
    seed: int


SHAPES = {
    "B": TransformerShape("B", 24, 1024, 16, 512, 30522, 2, 14, 2),
    "G": TransformerShape("G", 48, 1600, 25, 1024, 50257, 4, 36, 3),
}


class _Alloc:
    """Contiguous 2 MiB-aligned tensor layout in allocation order."""

    def __init__(self):
        self.next = 0
        self.tensors = {}

    def add(self, name: str, nbytes: int) -> None:
        nb = max(1, -(-nbytes // BLOCK_BYTES))
        self.tensors[name] = (self.next, nb)
        self.next += nb

    def blocks(self, name: str) -> List[int]:
        s, n = self.tensors[name]
        return list(range(s, s + n))


def _layout(sh: TransformerShape, b: int, workspace: int = 0) -> _Alloc:
    h, s, a, L, V = sh.hidden, sh.seq, sh.heads, sh.layers, sh.vocab
    al = _Alloc()
    weights = {"Wqkv": h * 3 * h, "Wo": h * h, "W1": h * 4 * h, "W2": 4 * h * h}
    for l in range(L):
        for w, n in weights.items():
            for part in ("p", "g", "m", "v"):       # fp32 master + grad + Adam m, v
                al.add(f"{w}.{part}.{l}", 4 * n)
        for ln in ("ln1", "ln2"):
            for part in ("p", "g", "m", "v"):
                al.add(f"{ln}.{part}.{l}", 4 * 2 * h)
    for part in ("p", "g", "m", "v"):
        al.add(f"emb.{part}", 4 * V * h)
    bsh = 2 * b * s * h                              # fp16 activations
    al.add("x.0", bsh)
    for l in range(L):
        for t in ("ln1_out", "ctx", "attn_out", "x2", "ln2_out", "h2"):
            al.add(f"{t}.{l}", bsh)
        al.add(f"x.{l + 1}", bsh)                   # x_next of layer l = x of layer l+1
        al.add(f"qkv.{l}", 3 * bsh)
        for t in ("scores", "probs", "probs_drop"):
            al.add(f"{t}.{l}", 2 * b * a * s * s)
        for t in ("h1", "gelu"):
            al.add(f"{t}.{l}", 4 * bsh)
    for i in range(3):
        al.add(f"gpool.{i}", 4 * bsh)               # reused activation-gradient buffers
    al.add("logits", 2 * b * s * V)
    al.add("loss", 4 * b * s)
    if workspace > 0:
        al.add("ws", workspace * BLOCK_BYTES)
    return al


def _interleave(*lists: Sequence[int]) -> List[int]:
    out: List[int] = []
    n = max(len(x) for x in lists)
    for i in range(n):
        for x in lists:
            if i < len(x):
                out.append(x[i])
    return out


def _kernels(sh: TransformerShape, al: _Alloc) -> List[Tuple[str, List[int]]]:
    L = sh.layers
    B = al.blocks
    has_ws = "ws" in al.tensors
    ws0 = [al.tensors["ws"][0]] if has_ws else []
    ks: List[Tuple[str, List[int]]] = []

    def k(name: str, tensors: Sequence[str], acc: List[int]):
        ks.append((f"{name}:" + ",".join(tensors), acc))

    def gemm(name, A, Bm, Cm, accumulate=False):
        acc = ws0 + _interleave(B(A), B(Bm)) + B(Cm)
        k(name, (A, Bm, Cm), acc)

    def ew(name, ins, out):
        acc = _interleave(*[B(t) for t in ins], B(out)) if out not in ins else _interleave(*[B(t) for t in ins])
        k(name, tuple(ins) + (out,), acc)

    def lnk(name, inp, w, out):
        k(name, (inp, w, out), B(inp) + B(w) + B(out))

    g = lambda i: f"gpool.{i % 3}"
    # ---- forward ----
    ew("emb_fwd", ["emb.p"], "x.0")
    for l in range(L):
        lnk(f"ln1_fwd.{l}", f"x.{l}", f"ln1.p.{l}", f"ln1_out.{l}")
        gemm(f"qkv_gemm.{l}", f"ln1_out.{l}", f"Wqkv.p.{l}", f"qkv.{l}")
        gemm(f"qk_gemm.{l}", f"qkv.{l}", f"qkv.{l}", f"scores.{l}")
        lnk(f"softmax.{l}", f"scores.{l}", f"scores.{l}", f"probs.{l}")
        ew(f"dropout_attn.{l}", [f"probs.{l}"], f"probs_drop.{l}")
        gemm(f"av_gemm.{l}", f"probs_drop.{l}", f"qkv.{l}", f"ctx.{l}")
        gemm(f"o_gemm.{l}", f"ctx.{l}", f"Wo.p.{l}", f"attn_out.{l}")
        ew(f"add1.{l}", [f"attn_out.{l}", f"x.{l}"], f"x2.{l}")
        lnk(f"ln2_fwd.{l}", f"x2.{l}", f"ln2.p.{l}", f"ln2_out.{l}")
        gemm(f"fc1_gemm.{l}", f"ln2_out.{l}", f"W1.p.{l}", f"h1.{l}")
        ew(f"gelu.{l}", [f"h1.{l}"], f"gelu.{l}")
        gemm(f"fc2_gemm.{l}", f"gelu.{l}", f"W2.p.{l}", f"h2.{l}")
        ew(f"add2.{l}", [f"h2.{l}", f"x2.{l}"], f"x.{l + 1}")
        ew(f"dropout_out.{l}", [f"x.{l + 1}"], f"x.{l + 1}")
    # ---- head: GEMM, 2 loss, 3 head bwd ----
    gemm("head_gemm", f"x.{L}", "emb.p", "logits")
    ew("loss_fwd", ["logits"], "loss")
    ew("loss_bwd", ["loss", "logits"], "logits")
    gemm("head_dgrad", "logits", "emb.p", g(0))
    gemm("head_wgrad", f"x.{L}", "logits", "emb.g")
    ew("head_bias_grad", ["logits"], "emb.g")
    # ---- backward: forward list reversed, 2 kernels per forward kernel ----
    gi = 0
    for l in reversed(range(L)):
        up, dn = g(gi), g(gi + 1)

        def bw_gemm(tag, A, W, Wgrad):
            nonlocal up, dn, gi
            gemm(f"{tag}_dgrad.{l}", up, W, dn)
            gemm(f"{tag}_wgrad.{l}", A, up, Wgrad)
            gi += 1
            up, dn = g(gi), g(gi + 1)

        def bw_ew(tag, saved: List[str], extra: str):
            nonlocal up, dn, gi
            ew(f"{tag}_grad.{l}", saved + [up], dn)
            ew(f"{tag}_red.{l}", [up], extra)
            gi += 1
            up, dn = g(gi), g(gi + 1)

        bw_ew("dropout_out", [f"x.{l + 1}"], dn)
        bw_ew("add2", [f"x2.{l}"], dn)
        bw_gemm("fc2", f"gelu.{l}", f"W2.p.{l}", f"W2.g.{l}")
        bw_ew("gelu", [f"h1.{l}"], dn)
        bw_gemm("fc1", f"ln2_out.{l}", f"W1.p.{l}", f"W1.g.{l}")
        bw_ew("ln2", [f"x2.{l}", f"ln2.p.{l}"], f"ln2.g.{l}")
        bw_ew("add1", [f"attn_out.{l}"], dn)
        bw_gemm("o", f"ctx.{l}", f"Wo.p.{l}", f"Wo.g.{l}")
        bw_gemm("av", f"probs_drop.{l}", f"qkv.{l}", up)
        bw_ew("dropout_attn", [f"probs.{l}"], dn)
        bw_ew("softmax", [f"probs.{l}"], dn)
        bw_gemm("qk", f"qkv.{l}", f"qkv.{l}", up)
        bw_gemm("qkv", f"ln1_out.{l}", f"Wqkv.p.{l}", f"Wqkv.g.{l}")
        bw_ew("ln1", [f"x.{l}", f"ln1.p.{l}"], f"ln1.g.{l}")
    ew("emb_bwd", [g(gi)], "emb.g")
    # ---- multi-tensor Adam over all parameters, in chunks ----
    params = [n for n in al.tensors if n.split(".")[1:2] == ["p"]]
    pblocks: List[Tuple[int, int, int, int]] = []
    for n in params:
        base = n.replace(".p", ".{}")
        for i in range(al.tensors[n][1]):
            pblocks.append(tuple(al.tensors[base.format(x)][0] + i for x in ("p", "g", "m", "v")))
    per = -(-len(pblocks) // sh.adam_chunks)
    for c in range(sh.adam_chunks):
        chunk = pblocks[c * per:(c + 1) * per]
        acc = [b for quad in chunk for b in quad]
        ks.append((f"adam.{c}", acc))
    return ks


def transformer_layout(sh: TransformerShape, C: int = HBM_FRAMES_B200):
    """Largest batch b with sum(blocks) <= oversub*C; the remainder becomes a
    workspace tensor so that W = oversub*C exactly."""
    target = sh.oversub * C
    lo, hi = 1, 1
    while _layout(sh, hi).next <= target:
        hi *= 2
    while hi - lo > 1:
        mid = (lo + hi) // 2
        if _layout(sh, mid).next <= target:
            lo = mid
        else:
            hi = mid
    b = lo
    used = _layout(sh, b).next
    al = _layout(sh, b, workspace=target - used)
    assert al.next == target, (al.next, target)
    return b, al


def make_transformer(which: str, n_iter: int = 10, seed: Optional[int] = None,
                     C: int = HBM_FRAMES_B200, jitter: float = 0.01, dup_ppm: int = 0) -> Trace:
    sh = SHAPES[which]
    seed = sh.seed if seed is None else seed
    b, al = transformer_layout(sh, C)
    ks = _kernels(sh, al)
    names = [n for n, _ in ks]
    offs = np.zeros(len(ks) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(a) for _, a in ks])
    acc = np.fromiter((x for _, a in ks for x in a), dtype=np.uint32, count=int(offs[-1]))
    W = al.next
    K = len(ks)
    base = np.array([fnv1a64(f"{which}:{n}".encode()) for n in names], dtype=np.uint64)
    hashes = _jitter_hashes(base, K, n_iter, seed, jitter)
    fo, fb, sb, sc = simulate_naive_um(W, C, offs, acc, n_iter, seed, dup_ppm)
    dead = []
    for n, (s0, nb) in al.tensors.items():
        stem = n.split(".")[0]
        if stem in ("Wqkv", "Wo", "W1", "W2", "ln1", "ln2", "emb"):
            continue
        dead.extend(range(s0, s0 + nb))
    tr = Trace(which, W, C, K, n_iter, hashes, fo, fb, sb, sc,
               np.array(sorted(dead), dtype=np.uint32), offs, acc, names, seed)
    tr.batch = b  # type: ignore[attr-defined]
    return tr


def make(config: str, n_iter: int = 10, seed: Optional[int] = None, **kw) -> Trace:
    if config == "T":
        return make_T(n_iter=n_iter, seed=1 if seed is None else seed, **kw)
    return make_transformer(config, n_iter=n_iter, seed=seed, **kw)


# ----------------------------------------------------------------------------
# Query streams and small random traces for tests
# ----------------------------------------------------------------------------
def random_trace(rng: np.random.Generator, n_launch: int, n_kernels: int, W: int,
                 max_faults: int, dup_prob: float = 0.2, empty_prob: float = 0.15):
    """Tiny random traces for brute-force checks: hashes drawn from a small
    pool of kernel names (so exec IDs repeat), random block lists with
    duplicates and empty launches."""
    pool = [fnv1a64(b"rk%d" % i) for i in range(n_kernels)]
    hashes = np.array([pool[int(rng.integers(n_kernels))] for _ in range(n_launch)], dtype=np.uint64)
    offs = [0]
    faults: List[int] = []
    for _ in range(n_launch):
        if rng.random() < empty_prob:
            offs.append(len(faults))
            continue
        n = int(rng.integers(1, max_faults + 1))
        lst = [int(x) for x in rng.integers(0, W, n)]
        for i in range(1, len(lst)):
            if rng.random() < dup_prob:
                lst[i] = lst[int(rng.integers(0, i))]
        faults += lst
        offs.append(len(faults))
    return hashes, np.array(offs, dtype=np.uint64), np.array(faults, dtype=np.uint32)
