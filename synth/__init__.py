"""Seeded synthetic workloads for the AutoPipe planner hot path.

This module is the ONLY code shared by the CUDA path and the oracle: it produces
input tables (per-sub-layer forward/backward nanoseconds and activation bytes) and
search parameters. It holds none of the method's arithmetic -- no stage sums, no
communication conversion, no simulation.

Workload recipe: a transformer is split at sub-layer
granularity into ``[embedding, (attention, ffn) x L, head]`` so ``n = 2L + 2``
(Fig. 3, "ResidualFFNBlocks and ResidualAttentionBlocks").
Per-sub-layer costs come from a GPT FLOP/byte model (activation checkpointing on,
PAPER.md:214, so backward = 3x forward for compute blocks):

* emb:  f = ceil(4*mbs*s*h / HBM_EFF),                 b = 2f
* attn: f = ceil((8*mbs*s*h^2 + 4*mbs*s^2*h) / R),      b = 3f
* ffn:  f = ceil(16*mbs*s*h^2 / R),                    b = 3f
* head: f = ceil(2*mbs*s*h*V / R),                     b = 2f
* act_bytes = 2*mbs*s*h (bf16) after every sub-layer except the head (0).

Constants: R = 700 000 FLOP/ns, HBM_EFF = 4 000 B/ns, link = 900e9 B/s.
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional, Tuple

import numpy as np

R_FLOP_PER_NS = 700_000
HBM_EFF_B_PER_NS = 4_000
LINK_BYTES_PER_S = 900_000_000_000


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


@dataclasses.dataclass(frozen=True)
class Workload:
    """One BASELINE.json config: tables + search parameters."""

    name: str
    fwd_ns: Tuple[int, ...]
    bwd_ns: Tuple[int, ...]
    act_bytes: Tuple[int, ...]
    link_bytes_per_s: int
    p: int
    m: int
    k_lo: int
    k_hi: int
    search: str  # "exhaustive" | "heuristic"
    restarts: int = 0
    seed: int = 0x5EED
    radius: int = 2
    slice_k_max: int = 0

    @property
    def n(self) -> int:
        return len(self.fwd_ns)

    def arrays(self):
        """int64 numpy copies of (fwd_ns, bwd_ns, act_bytes)."""
        return (np.asarray(self.fwd_ns, dtype=np.int64),
                np.asarray(self.bwd_ns, dtype=np.int64),
                np.asarray(self.act_bytes, dtype=np.int64))


def gpt_tables(L: int, h: int, s: int, mbs: int, V: int):
    """Per-sub-layer (fwd_ns, bwd_ns, act_bytes) lists for a GPT of L layers."""
    f: List[int] = []
    b: List[int] = []
    a: List[int] = []
    act = 2 * mbs * s * h
    fe = _ceil_div(4 * mbs * s * h, HBM_EFF_B_PER_NS)
    f.append(fe); b.append(2 * fe); a.append(act)
    fa = _ceil_div(8 * mbs * s * h * h + 4 * mbs * s * s * h, R_FLOP_PER_NS)
    ff = _ceil_div(16 * mbs * s * h * h, R_FLOP_PER_NS)
    for _ in range(L):
        f.append(fa); b.append(3 * fa); a.append(act)
        f.append(ff); b.append(3 * ff); a.append(act)
    fh = _ceil_div(2 * mbs * s * h * V, R_FLOP_PER_NS)
    f.append(fh); b.append(2 * fh); a.append(0)
    return f, b, a


def gpt_memory(L: int, h: int, s: int, mbs: int, V: int):
    """Per-sub-layer (static_bytes, stash_bytes) for the N4 memory model (DESIGN.md
    reading R-N4), same sub-layer order as gpt_tables.

    static: 16 B per parameter (bf16 weight + bf16 gradient + fp32 master weight + two
    fp32 Adam moments); parameters: emb V*h + s*h, attn 4h^2 + 4h + 2h (LayerNorm),
    ffn 8h^2 + 5h + 2h, head V*h + 2h (untied).
    stash (activation checkpointing): the sub-layer's input per in-flight
    micro-batch -- token ids (8 B each) for emb, the bf16 hidden state 2*mbs*s*h else."""
    st: List[int] = []
    sh: List[int] = []
    hid = 2 * mbs * s * h
    st.append(16 * (V * h + s * h)); sh.append(8 * mbs * s)
    for _ in range(L):
        st.append(16 * (4 * h * h + 6 * h)); sh.append(hid)
        st.append(16 * (8 * h * h + 7 * h)); sh.append(hid)
    st.append(16 * (V * h + 2 * h)); sh.append(hid)
    return st, sh


@dataclasses.dataclass(frozen=True)
class DepthWorkload:
    """NEXT N4: outer planner loop over pipeline depth with a memory model."""

    name: str
    base: Workload           # tables (its p, m are unused)
    static_bytes: Tuple[int, ...]
    stash_bytes: Tuple[int, ...]
    cap_bytes: int
    n_gpus: int
    microbatches: int        # per iteration, over all data-parallel replicas


def depth_config() -> DepthWorkload:
    """GPT-2 1.3B (Table I: 24 layers, h 2048) with micro-batch size 16 on 8
    GPUs, global batch 512 (Table IV) -> 32 micro-batches per iteration; per-GPU
    capacity 24 GiB (the paper's RTX 3090s)."""
    L, h, s, mbs, V = 24, 2048, 1024, 16, 50257
    f, b, a = gpt_tables(L, h, s, mbs, V)
    base = Workload(name="N4-gpt2-1.3b-mbs16", fwd_ns=tuple(f), bwd_ns=tuple(b),
                    act_bytes=tuple(a), link_bytes_per_s=LINK_BYTES_PER_S, p=1, m=1,
                    k_lo=1, k_hi=1, search="exhaustive")
    st, sh = gpt_memory(L, h, s, mbs, V)
    return DepthWorkload(name="N4-gpt2-1.3b-mbs16-g8-gbs512-24GiB", base=base,
                         static_bytes=tuple(st), stash_bytes=tuple(sh), cap_bytes=24 << 30,
                         n_gpus=8, microbatches=512 // mbs)


def _wl(name, L, h, s, mbs, V, **kw) -> Workload:
    f, b, a = gpt_tables(L, h, s, mbs, V)
    return Workload(name=name, fwd_ns=tuple(f), bwd_ns=tuple(b), act_bytes=tuple(a),
                    link_bytes_per_s=LINK_BYTES_PER_S, **kw)


def config(idx: int) -> Workload:
    """BASELINE.json configs[idx-1] (1-based C1..C5)."""
    if idx == 1:   # tiny 4-layer GPT, p=4, m=8, exhaustive 84 candidates, no slicing
        return _wl("C1-tiny-gpt-n10-p4-m8", 4, 256, 256, 1, 8192,
                   p=4, m=8, k_lo=1, k_hi=1, search="exhaustive")
    if idx == 2:   # GPT-2-medium shaped, p=4, m=16, k in 1..4
        return _wl("C2-gpt2-medium-n50-p4-m16-k4", 24, 1024, 1024, 4, 50257,
                   p=4, m=16, k_lo=1, k_hi=4, search="exhaustive")
    if idx == 3:   # 24-layer GPT, p=8, m=32
        return _wl("C3-gpt24-n50-p8-m32", 24, 1024, 1024, 4, 50257,
                   p=8, m=32, k_lo=1, k_hi=1, search="exhaustive")
    if idx == 4:   # GPT-3-2.7B shaped, p=8, m=64, k in 1..8
        return _wl("C4-gpt3-2.7b-n66-p8-m64-k8", 32, 2560, 2048, 1, 50257,
                   p=8, m=64, k_lo=1, k_hi=8, search="exhaustive")
    if idx == 5:   # 48-layer GPT, p=16, m=64, heuristic 65536 restarts + slice sweep K=16
        return _wl("C5-gpt48-n98-p16-m64-heur65536", 48, 1600, 1024, 4, 50257,
                   p=16, m=64, k_lo=1, k_hi=1, search="heuristic", restarts=65536,
                   seed=0x5EED, radius=2, slice_k_max=16)
    raise ValueError(f"no config C{idx}")


ALL_CONFIGS = (1, 2, 3, 4, 5)


def random_tables(seed: int, n: int, kind: str = "uniform",
                  fmax: int = 1 << 20, amax: int = 1 << 27):
    """Seeded random (fwd_ns, bwd_ns, act_bytes) int64 arrays for property tests.

    kinds: "uniform" (U[0,fmax] ns, U[0,amax] bytes), "zero" (all zero),
    "equal" (all blocks identical -> many ties), "huge" (uniform plus one head-like
    block 6x the max), "small" (U[0,7] ns, U[0,3] bytes with bw=1e9 -> dense ties),
    "b3f" (b = 3f like checkpointed compute blocks).
    """
    rng = np.random.default_rng(seed)
    if kind == "zero":
        f = np.zeros(n, np.int64); b = np.zeros(n, np.int64); a = np.zeros(n, np.int64)
    elif kind == "equal":
        v = int(rng.integers(0, fmax + 1)); w = int(rng.integers(0, fmax + 1))
        f = np.full(n, v, np.int64); b = np.full(n, w, np.int64)
        a = np.full(n, int(rng.integers(0, amax + 1)), np.int64)
    elif kind == "small":
        f = rng.integers(0, 8, n).astype(np.int64); b = rng.integers(0, 8, n).astype(np.int64)
        a = rng.integers(0, 4, n).astype(np.int64)
    elif kind == "b3f":
        f = rng.integers(0, fmax + 1, n).astype(np.int64); b = 3 * f
        a = rng.integers(0, amax + 1, n).astype(np.int64)
    else:
        f = rng.integers(0, fmax + 1, n).astype(np.int64)
        b = rng.integers(0, fmax + 1, n).astype(np.int64)
        a = rng.integers(0, amax + 1, n).astype(np.int64)
        if kind == "huge":
            j = int(rng.integers(0, n))
            f[j] = 6 * fmax; b[j] = 12 * fmax
        elif kind != "uniform":
            raise ValueError(kind)
    return f, b, a


def random_cuts(seed: int, n: int, p: int, count: int) -> np.ndarray:
    """`count` uniformly random valid cut vectors int32[count, p-1] (strictly
    increasing in [1, n-1]), seeded."""
    rng = np.random.default_rng(seed)
    out = np.zeros((count, max(p - 1, 0)), np.int32)
    for i in range(count):
        if p > 1:
            out[i] = np.sort(rng.choice(np.arange(1, n), size=p - 1, replace=False))
    return out


def link_for(kind: str) -> int:
    """Link bandwidth paired with a random table kind."""
    return 1_000_000_000 if kind == "small" else LINK_BYTES_PER_S
