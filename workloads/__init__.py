"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module holds INPUTS only: per-layer profiles (Table 1 rows O, G, P), cluster
states (Table 1 rows N, B, FP, BP) and partition records. It contains none of the
cost model's arithmetic (no stage sums, transfers, all-reduce or recurrence). Converting a
workload's FLOPs into nanoseconds and a NIC speed into femtoseconds per byte is how the inputs are
*made*; both sides receive the result.

Everything is deterministic: fixed tables, or numpy ``default_rng`` with the seeds of App. B.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import List, Optional, Sequence

import numpy as np

U64_MAX = (1 << 64) - 1
IDLE = 0xFF

# rates used to turn shapes into times (App. B): P100-like fp32 (the paper's testbed,
# PAPER.md:1070-1071) and half of the measured B200 bf16 sustained rate for BERT/GPT.
P100_FLOP_PER_NS = 4650
P100_BYTES_PER_NS = 732
B200_FLOP_PER_NS = 676_000
B200_BYTES_PER_NS = 6552

GBPS = {10: 800_000, 25: 320_000, 40: 200_000, 50: 160_000, 100: 80_000}
NVLINK5_FS_PER_BYTE = 1112  # ceil(1e15 / 9e11)


def fs_per_byte(gbit_per_s: float) -> int:
    """Inverse bandwidth in fs/B for a link of ``gbit_per_s`` (reading C-5): ceil(8e15 / bit/s)."""
    bits = int(round(gbit_per_s * 1e9))
    return -(-8 * 10**15 // bits)


@dataclass
class Profile:
    """Static metrics of Table 1."""
    name: str
    O: List[int]            # output activation bytes per layer
    G: List[int]            # bytes of the gradient w.r.t. the layer input
    P: List[int]            # weight bytes
    f_ref: List[int]        # forward ns on an uncontended reference worker
    b_ref: List[int]        # backward ns on an uncontended reference worker

    @property
    def L(self) -> int:
        return len(self.O)

    def arrays(self):
        return (np.asarray(self.O, dtype=np.uint64), np.asarray(self.G, dtype=np.uint64),
                np.asarray(self.P, dtype=np.uint64))


@dataclass
class State:
    """Dynamic metrics of Table 1: N workers, FP/BP (N x L ns), link tau (N x N fs/B)."""
    f: List[List[int]]
    b: List[List[int]]
    tau: List[List[int]]
    label: str = ""

    @property
    def N(self) -> int:
        return len(self.f)

    def arrays(self):
        return (np.asarray(self.f, dtype=np.uint64), np.asarray(self.b, dtype=np.uint64),
                np.asarray(self.tau, dtype=np.uint64))


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


# --------------------------------------------------------------------------------------------
# Profiles (App. B.1 - B.6)
# --------------------------------------------------------------------------------------------

def toy() -> Profile:
    """C1 (App. B.1): 8-layer chain; f = [1,2,3,4,4,3,2,1] ms, b = 2f."""
    f = [v * 10**6 for v in (1, 2, 3, 4, 4, 3, 2, 1)]
    O = [8_000_000, 8_000_000, 4_000_000, 4_000_000, 2_000_000, 2_000_000, 1_000_000, 4_000]
    G = [0] + O[:-1]
    P = [v * 10**6 for v in (1, 1, 2, 2, 4, 4, 8, 8)]
    return Profile("toy", O, G, P, f, [2 * x for x in f])


def vgg16(batch: int = 64) -> Profile:
    """C2 (App. B.2): VGG-16 at 224x224, fp32, 21 layer groups (13 conv, 5 pool, 3 fc)."""
    cfg = [("conv", 3, 64, 224), ("conv", 64, 64, 224), ("pool", 64, 112),
           ("conv", 64, 128, 112), ("conv", 128, 128, 112), ("pool", 128, 56),
           ("conv", 128, 256, 56), ("conv", 256, 256, 56), ("conv", 256, 256, 56), ("pool", 256, 28),
           ("conv", 256, 512, 28), ("conv", 512, 512, 28), ("conv", 512, 512, 28), ("pool", 512, 14),
           ("conv", 512, 512, 14), ("conv", 512, 512, 14), ("conv", 512, 512, 14), ("pool", 512, 7),
           ("fc", 25088, 4096), ("fc", 4096, 4096), ("fc", 4096, 1000)]
    O, P, f = [], [], []
    for c in cfg:
        if c[0] == "conv":
            _, ci, co, h = c
            P.append(4 * (9 * ci * co + co))
            O.append(co * h * h * batch * 4)
            f.append(_ceil_div(2 * 9 * ci * co * h * h * batch, P100_FLOP_PER_NS))
        elif c[0] == "pool":
            _, ch, h = c
            out = ch * h * h
            P.append(0)
            O.append(out * batch * 4)
            f.append(_ceil_div(5 * out * batch * 4, P100_BYTES_PER_NS))
        else:
            _, i, o = c
            P.append(4 * (i * o + o))
            O.append(o * batch * 4)
            f.append(_ceil_div(2 * i * o * batch, P100_FLOP_PER_NS))
    G = [3 * 224 * 224 * batch * 4] + O[:-1]
    return Profile("vgg16", O, G, P, f, [2 * x for x in f])


def resnet50(batch: int = 128) -> Profile:
    """C5 (App. B.3): ResNet-50, one layer per conv (conv1+maxpool, 16 bottlenecks x 3, fc), fp32.

    Cuts inside a bottleneck also carry the block input (the skip tensor), so O of the first two
    convs of a block includes it; the downsample projection is folded into the block's third conv.
    """
    O, P, f = [], [], []
    # conv1 7x7/2 3->64 at 112, then maxpool to 56
    P.append(4 * 7 * 7 * 3 * 64)
    f.append(_ceil_div(2 * 7 * 7 * 3 * 64 * 112 * 112 * batch, P100_FLOP_PER_NS)
             + _ceil_div(5 * 64 * 56 * 56 * batch * 4, P100_BYTES_PER_NS))
    O.append(64 * 56 * 56 * batch * 4)
    cin, hw = 64, 56
    for n_blocks, mid, out, stride in ((3, 64, 256, 1), (4, 128, 512, 2), (6, 256, 1024, 2),
                                       (3, 512, 2048, 2)):
        for blk in range(n_blocks):
            s = stride if blk == 0 else 1
            h_in, h_out = hw, hw // s
            skip = cin * h_in * h_in * batch * 4
            # 1x1 reduce (stride applied here, ResNet v1.5 puts it on the 3x3; shapes are what matter)
            P.append(4 * cin * mid)
            f.append(_ceil_div(2 * cin * mid * h_in * h_in * batch, P100_FLOP_PER_NS))
            O.append(mid * h_in * h_in * batch * 4 + skip)
            # 3x3
            P.append(4 * 9 * mid * mid)
            f.append(_ceil_div(2 * 9 * mid * mid * h_out * h_out * batch, P100_FLOP_PER_NS))
            O.append(mid * h_out * h_out * batch * 4 + skip)
            # 1x1 expand (+ projection on the first block)
            proj_p = cin * out if blk == 0 else 0
            P.append(4 * (mid * out + proj_p))
            f.append(_ceil_div(2 * (mid * out + proj_p) * h_out * h_out * batch, P100_FLOP_PER_NS))
            O.append(out * h_out * h_out * batch * 4)
            cin, hw = out, h_out
    # avgpool + fc 2048 -> 1000
    P.append(4 * (2048 * 1000 + 1000))
    f.append(_ceil_div(2 * 2048 * 1000 * batch, P100_FLOP_PER_NS)
             + _ceil_div(2048 * 7 * 7 * batch * 4, P100_BYTES_PER_NS))
    O.append(1000 * batch * 4)
    G = [3 * 224 * 224 * batch * 4] + O[:-1]
    return Profile("resnet50", O, G, P, f, [2 * x for x in f])


def gnmt16(batch: int = 64, seq: int = 50, h: int = 1024, vocab: int = 32000) -> Profile:
    """C3 (App. B.4): GNMT-16 (embedding, 8 encoder LSTMs, 8 decoder LSTMs, classifier), fp32."""
    tok = batch * seq
    O, P, f = [], [], []
    P.append(vocab * h * 4); O.append(tok * h * 4); f.append(_ceil_div(tok * h * 4, P100_BYTES_PER_NS))
    for _ in range(8):
        P.append(4 * (2 * h) * h * 4)
        O.append(tok * h * 4)
        f.append(_ceil_div(2 * 4 * (2 * h) * h * tok, P100_FLOP_PER_NS))
    for i in range(8):
        att_p = h * 2 * h * 4 if i == 0 else 0
        P.append(4 * (3 * h) * h * 4 + att_p)
        O.append(2 * tok * h * 4)                     # hidden + attention context
        att_f = _ceil_div(2 * h * 2 * h * tok, P100_FLOP_PER_NS) if i == 0 else 0
        f.append(_ceil_div(2 * 4 * (3 * h) * h * tok, P100_FLOP_PER_NS) + att_f)
    P.append(vocab * h * 4); O.append(0); f.append(_ceil_div(2 * h * vocab * tok, P100_FLOP_PER_NS))
    G = [0] + O[:-1]
    return Profile("gnmt16", O, G, P, f, [2 * x for x in f])


def bert24(mb: int = 8, seq: int = 512, d: int = 1024, vocab: int = 30522) -> Profile:
    """C3 (App. B.5): BERT-24 (embedding, 24 blocks, MLM head), bf16, B200 rates."""
    tok = mb * seq
    act = tok * d * 2
    O, P, f = [act], [vocab * d * 2], [_ceil_div(act, B200_BYTES_PER_NS)]
    for _ in range(24):
        P.append((12 * d * d + 13 * d) * 2)
        O.append(act)
        f.append(_ceil_div(24 * tok * d * d + 4 * mb * seq * seq * d, B200_FLOP_PER_NS))
    P.append(0); O.append(0); f.append(_ceil_div(2 * tok * d * vocab, B200_FLOP_PER_NS))
    G = [0] + O[:-1]
    return Profile("bert24", O, G, P, f, [2 * x for x in f])


def gpt96(seed: int = 96, d: int = 12288, seq: int = 2048, vocab: int = 50257) -> Profile:
    """C4 (App. B.6): 96-layer GPT-3-shaped transformer, mb 1, bf16, per-layer jitter U[0.95,1.05]."""
    rng = np.random.default_rng(seed)
    jitter = rng.integers(950, 1051, size=96).tolist()
    f_base = _ceil_div(24 * seq * d * d + 4 * seq * seq * d, B200_FLOP_PER_NS)
    act = seq * d * 2
    f = [_ceil_div(f_base * j, 1000) for j in jitter]
    P = [12 * d * d * 2] * 96
    emb = vocab * d * 2
    P[0] += emb
    P[95] += emb
    f[95] += _ceil_div(2 * seq * d * vocab, B200_FLOP_PER_NS)
    O = [act] * 96
    G = [act] * 96
    return Profile("gpt96", O, G, P, f, [2 * x for x in f])


PROFILES = {"toy": toy, "vgg16": vgg16, "resnet50": resnet50, "gnmt16": gnmt16,
            "bert24": bert24, "gpt96": gpt96}


def profile(name: str) -> Profile:
    return PROFILES[name]()


# --------------------------------------------------------------------------------------------
# States (App. B, B.7)
# --------------------------------------------------------------------------------------------

def make_state(prof: Profile, slowdown: Sequence[int], nic_gbps: Optional[Sequence[float]] = None,
               tau: Optional[Sequence[Sequence[int]]] = None, label: str = "") -> State:
    """Worker w runs every layer ``slowdown[w]`` times slower (k co-located jobs).

    Links: either an explicit tau matrix, or per-worker NIC speeds with tau[u][v] from the slower
    NIC (reading C-5)."""
    N = len(slowdown)
    f = [[x * k for x in prof.f_ref] for k in slowdown]
    b = [[x * k for x in prof.b_ref] for k in slowdown]
    if tau is None:
        t = [fs_per_byte(g) for g in nic_gbps]
        tau = [[0 if u == v else max(t[u], t[v]) for v in range(N)] for u in range(N)]
    return State(f, b, [list(r) for r in tau], label)


def uniform_state(prof: Profile, N: int, fs: int, label: str = "") -> State:
    tau = [[0 if u == v else fs for v in range(N)] for u in range(N)]
    return make_state(prof, [1] * N, tau=tau, label=label)


def toy_state() -> State:
    """C1: 4 identical workers, uniform 10 Gb/s (tau = 800000 fs/B)."""
    return uniform_state(toy(), 4, GBPS[10], "toy-10G")


def vgg_state(seed: int = 1) -> State:
    """C2: 8 workers, per-worker NIC speed drawn from {10,25,40,100} Gb/s with seed 1."""
    rng = np.random.default_rng(seed)
    nic = rng.choice([10, 25, 40, 100], size=8).tolist()
    return make_state(vgg16(), [1] * 8, nic_gbps=nic, label=f"vgg-nic{nic}")


def gpt_state(kind: str = "a-nvlink") -> State:
    """C4a: homogeneous 8 workers on NVLink 5 or 100 Gb/s; C4b: workers 5-6 x2, link 3->4 at 25 Gb/s."""
    prof = gpt96()
    if kind == "a-nvlink":
        return uniform_state(prof, 8, NVLINK5_FS_PER_BYTE, "C4a-nvlink")
    if kind == "a-100g":
        return uniform_state(prof, 8, GBPS[100], "C4a-100G")
    if kind == "b":
        tau = [[0 if u == v else GBPS[100] for v in range(8)] for u in range(8)]
        tau[3][4] = GBPS[25]
        return make_state(prof, [1, 1, 1, 1, 1, 2, 2, 1], tau=tau, label="C4b")
    raise ValueError(kind)


# App. B.7: the C3 trace, one row per state switch: (N, slowdown per worker, NIC Gb/s per worker)
TRACE_C3 = [
    ("exclusive start", [1] * 8, [100] * 8),
    ("bandwidth halved (E1)", [1] * 8, [50] * 8),
    ("Fig. 9 step 10G", [1] * 8, [10] * 8),
    ("Fig. 9 step 25G", [1] * 8, [25] * 8),
    ("Fig. 9 step 40G", [1] * 8, [40] * 8),
    ("Fig. 9 step 100G", [1] * 8, [100] * 8),
    ("+1 job on every GPU (E2)", [2] * 8, [100] * 8),
    ("+1 more job on workers 0-3", [3, 3, 3, 3, 2, 2, 2, 2], [100] * 8),
    ("jobs finish (E4)", [1] * 8, [100] * 8),
    ("new distributed job takes 2 GPUs (E3)", [1] * 6, [40, 40, 40, 100, 100, 100]),
    ("contention on remaining GPUs", [2, 2, 1, 1, 1, 1], [40, 40, 40, 100, 100, 100]),
    ("other job finishes (E4)", [1] * 8, [100] * 8),
]


def trace_c3(prof: Profile) -> List[State]:
    return [make_state(prof, k, nic_gbps=nic, label=lab) for lab, k, nic in TRACE_C3]


def rollout_state(prof: Profile, step: int) -> State:
    """C5: per step (seed 1000 + step) N_avail in {4..8}, slowdowns in {1,2,3}, NIC in {10,25,40,100}."""
    rng = np.random.default_rng(1000 + step)
    N = int(rng.integers(4, 9))
    k = rng.integers(1, 4, size=N).tolist()
    nic = rng.choice([10, 25, 40, 100], size=N).tolist()
    return make_state(prof, k, nic_gbps=nic, label=f"rollout-step{step}")


def testbed_state(prof: Profile, seed: int = 10, N: int = 10) -> State:
    """NEXT f4: the paper's testbed size, 10 GPUs with per-GPU NIC speeds from
    {10, 25, 40, 100} Gb/s (its network settings) and slowdowns in {1, 2} (co-located jobs), seeded."""
    rng = np.random.default_rng(seed)
    k = rng.integers(1, 3, size=N).tolist()
    nic = rng.choice([10, 25, 40, 100], size=N).tolist()
    return make_state(prof, k, nic_gbps=nic, label=f"testbed{N}-seed{seed}")


def random_state(prof: Profile, N: int, rng: np.random.Generator, max_slow: int = 3,
                 free_link_p: float = 0.0) -> State:
    """A random heterogeneous state: per-worker slowdown, per-directed-link speed (asymmetric)."""
    k = rng.integers(1, max_slow + 1, size=N).tolist()
    choices = [GBPS[10], GBPS[25], GBPS[40], GBPS[100], NVLINK5_FS_PER_BYTE]
    tau = [[0] * N for _ in range(N)]
    for u in range(N):
        for v in range(N):
            if u != v:
                tau[u][v] = 0 if rng.random() < free_link_p else int(rng.choice(choices))
    return make_state(prof, k, tau=tau)


def random_profile(L: int, rng: np.random.Generator, f_max: int = 1000, bytes_max: int = 10**6,
                   zero_p: float = 0.1) -> Profile:
    """Small random profiles for parity and oracle pins (independent f and b, some zeros)."""
    def draw(hi):
        v = rng.integers(0, hi + 1, size=L)
        v[rng.random(L) < zero_p] = 0
        return [int(x) for x in v]
    return Profile(f"rand{L}", draw(bytes_max), draw(bytes_max), draw(bytes_max),
                   draw(f_max), draw(2 * f_max))


def random_state_small(prof: Profile, N: int, rng: np.random.Generator, tau_max: int = 2000) -> State:
    """Random per-worker f/b (independent per worker and layer) and random tau, for tiny pins."""
    L = prof.L
    f = [[int(x) for x in rng.integers(0, 1000, size=L)] for _ in range(N)]
    b = [[int(x) for x in rng.integers(0, 2000, size=L)] for _ in range(N)]
    tau = [[0 if u == v else int(rng.integers(0, tau_max + 1)) for v in range(N)] for u in range(N)]
    return State(f, b, tau, "random-small")


# --------------------------------------------------------------------------------------------
# Partition records (SPEC.md §2): 16 bytes = S, last_layer[7], stage_of_worker[8]
# --------------------------------------------------------------------------------------------

def encode(S: int, cuts: Sequence[int], stage_of_worker: Sequence[int], wide: bool = False) -> bytes:
    """16-byte record, or the 32-byte wide record (S, last_layer[15], stage_of_worker[16]; NEXT f4)."""
    n, off = (32, 16) if wide else (16, 8)
    rec = bytearray([IDLE] * n)
    rec[0] = S
    for i, e in enumerate(cuts):
        rec[1 + i] = e
    for w, s in enumerate(stage_of_worker):
        rec[off + w] = s
    return bytes(rec)


def contiguous_record(L: int, cuts: Sequence[int], sizes: Sequence[int], wide: bool = False) -> bytes:
    """Stage s gets the next sizes[s] workers in state order."""
    sow, w = [], 0
    for s, r in enumerate(sizes):
        sow += [s] * r
    return encode(len(sizes), cuts, sow, wide)


def sample_records(L: int, N: int, count: int, seed: int, random_placement_p: float = 0.5,
                   s_max: int = 8, wide: bool = False) -> np.ndarray:
    """C5 record sampler (App. B): S ~ U{1..min(s_max,N)}, uniform cut set, uniform composition with
    sum r <= N, contiguous placement in (1-p) of the records and a random worker permutation in p.

    Returns a (count, 16) uint8 array, or (count, 32) wide records (S <= 16, N <= 16; NEXT f4).
    Vectorised per S; seeded with ``numpy.random.default_rng``.
    """
    rng = np.random.default_rng(seed)
    width, off = (32, 16) if wide else (16, 8)
    if not wide and (s_max > 8 or N > 8):
        raise ValueError("16-byte records hold S <= 8 and N <= 8; use wide=True")
    out = np.full((count, width), IDLE, dtype=np.uint8)
    smax = min(s_max, N, L)
    S = rng.integers(1, smax + 1, size=count)
    out[:, 0] = S
    for s in range(1, smax + 1):
        idx = np.nonzero(S == s)[0]
        n = idx.size
        if n == 0:
            continue
        if s > 1:
            cuts = np.sort(np.argsort(rng.random((n, L - 1)), axis=1)[:, :s - 1], axis=1)
            out[idx, 1:s] = cuts.astype(np.uint8)
        # composition: R_1 < ... < R_S an s-subset of {1..N}
        R = np.sort(np.argsort(rng.random((n, N)), axis=1)[:, :s], axis=1) + 1
        Rprev = np.concatenate([np.zeros((n, 1), dtype=R.dtype), R[:, :-1]], axis=1)
        pos = np.arange(N)[None, :]
        stage = np.full((n, N), IDLE, dtype=np.int64)
        for t in range(s):
            m = (pos >= Rprev[:, t:t + 1]) & (pos < R[:, t:t + 1])
            stage[m] = t
        perm_rows = rng.random(n) < random_placement_p
        perms = np.argsort(rng.random((n, N)), axis=1)
        shuffled = np.take_along_axis(stage, perms, axis=1)
        stage = np.where(perm_rows[:, None], shuffled, stage)
        out[idx, off:off + N] = stage.astype(np.uint8)
    return out


def r1_records(L: int, S: int, count: int, seed: int) -> np.ndarray:
    """`count` 16-byte records of S stages with one worker each (stage s on worker s) and a uniform
    random cut set: the S = 8, r = 1 candidates the SURVEY's 230-op full-T unit describes. Chunked so
    the random keys stay small."""
    rng = np.random.default_rng(seed)
    out = np.full((count, 16), IDLE, dtype=np.uint8)
    out[:, 0] = S
    out[:, 8:8 + S] = np.arange(S, dtype=np.uint8)
    step = 1 << 16
    for a in range(0, count, step):
        n = min(step, count - a)
        keys = rng.random((n, L - 1), dtype=np.float32)
        cuts = np.sort(np.argpartition(keys, S - 1, axis=1)[:, :S - 1], axis=1)
        out[a:a + n, 1:S] = cuts.astype(np.uint8)
    return out


def corrupt_records(recs: np.ndarray, L: int, N: int, seed: int, frac: float = 0.2) -> np.ndarray:
    """Mutate a fraction of records with random field edits (some stay valid, most become invalid)."""
    rng = np.random.default_rng(seed)
    out = recs.copy()
    MS = 16 if out.shape[1] == 32 else 8
    rows = np.nonzero(rng.random(len(out)) < frac)[0]
    for r in rows:
        kind = int(rng.integers(0, 6))
        if kind == 0:
            out[r, 0] = int(rng.choice([0, MS + 1, 255, min(MS, N) + 1]))
        elif kind == 1:
            out[r, 1 + int(rng.integers(0, MS - 1))] = int(rng.integers(0, 256))
        elif kind == 2:
            out[r, MS + int(rng.integers(0, MS))] = int(rng.integers(0, 256))
        elif kind == 3:
            out[r, MS + int(rng.integers(0, MS))] = IDLE
        elif kind == 4:
            out[r, 1] = L - 1
        else:
            out[r, MS + int(rng.integers(0, MS))] = int(rng.integers(0, MS))
    return out
