"""Oracle: the ingredients of the schedule (SPEC.md §2-3). Test infrastructure only.

Everything is exact Python integers. Each function cites the passage it follows.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Sequence, Tuple

IDLE = 0xFF
U64_MAX = (1 << 64) - 1


def ceil_div(a: int, b: int) -> int:
    return -(-a // b)


@dataclass
class Partition:
    """A worker partition: S stages, their last layers, their worker sets."""
    S: int
    cuts: List[int]          # e_0 < ... < e_{S-2}
    W: List[List[int]]       # W[s] ascending worker ids

    def stage_layers(self, L: int) -> List[Tuple[int, int]]:
        """[a_s, e_s] per stage, a_0 = 0, e_{S-1} = L-1, a_{s+1} = e_s + 1 (SPEC §2)."""
        ends = list(self.cuts) + [L - 1]
        out, a = [], 0
        for e in ends:
            out.append((a, e))
            a = e + 1
        return out


def parse_record(rec: bytes, L: int, N: int) -> Optional[Partition]:
    """Decode a 16-byte record (SPEC §2) or a 32-byte wide record (NEXT row f4: S <= 16 stages,
    N <= 16 workers, for the paper's 10-GPU testbed). Returns None if invalid.

    16 bytes: S, last_layer[7], stage_of_worker[8]; 32 bytes: S, last_layer[15], stage_of_worker[16].
    Invalid iff: S not in [1, min(MS, N)] (MS = 8 or 16); first S-1 cuts not strictly increasing or
    not < L-1; a stage without a worker; a worker >= N with a stage; a stage id not in [0,S) or 0xFF.
    """
    rec = bytes(rec)
    if len(rec) == 16:
        MS, off = 8, 8
    elif len(rec) == 32:
        MS, off = 16, 16
    else:
        raise ValueError("a partition record has 16 or 32 bytes")
    S = rec[0]
    if not (1 <= S <= min(MS, N)):
        return None
    cuts = list(rec[1:S])
    prev = -1
    for e in cuts:
        if e <= prev or e >= L - 1:
            return None
        prev = e
    W: List[List[int]] = [[] for _ in range(S)]
    for w in range(MS):
        s = rec[off + w]
        if s == IDLE:
            continue
        if w >= N or s >= S:
            return None
        W[s].append(w)
    if any(len(ws) == 0 for ws in W):
        return None
    return Partition(S, cuts, W)


def encode_partition(p: Partition, wide: bool = False) -> bytes:
    """The 16-byte record of p, or its 32-byte wide record (needed when S > 8 or a worker >= 8)."""
    n, off = (32, 16) if wide else (16, 8)
    rec = bytearray([IDLE] * n)
    rec[0] = p.S
    for i, e in enumerate(p.cuts):
        rec[1 + i] = e
    for s, ws in enumerate(p.W):
        for w in ws:
            rec[off + w] = s
    return bytes(rec)


def xfer(nbytes: int, fs_per_byte: int) -> int:
    """Transfer time in ns: ceil(bytes * tau / 1e6) (SPEC §1, reading C-7)."""
    return ceil_div(nbytes * fs_per_byte, 10**6)


def shards(A: int, r: int) -> List[Tuple[int, int]]:
    """Byte range held by replica i of a split stage: [floor(iA/r), floor((i+1)A/r)) (SPEC §3)."""
    return [(i * A // r, (i + 1) * A // r) for i in range(r)]


def boundary_transfers(A: int, senders: Sequence[int], receivers: Sequence[int],
                       tau: Sequence[Sequence[int]]) -> List[Tuple[int, int, int]]:
    """Transfers of one stage boundary: every (sender i, receiver j) whose shards overlap by ov > 0
    is one transfer on the directed link senders[i] -> receivers[j] lasting xfer(ov) (SPEC §3;
    p2p activations / gradients). Returns (u, v, duration) triples."""
    out = []
    S_sh = shards(A, len(senders))
    R_sh = shards(A, len(receivers))
    for i, (lo_i, hi_i) in enumerate(S_sh):
        for j, (lo_j, hi_j) in enumerate(R_sh):
            ov = min(hi_i, hi_j) - max(lo_i, lo_j)
            if ov > 0:
                u, v = senders[i], receivers[j]
                out.append((u, v, xfer(ov, tau[u][v])))
    return out


@dataclass
class Ingredients:
    """Per-op durations of one partition under one state (SPEC §2-3)."""
    S: int
    W: List[List[int]]
    Fd: List[dict]                      # Fd[s][w] = F'_{s,w}
    Bd: List[dict]                      # Bd[s][w] = B'_{s,w}
    fwd: List[List[Tuple[int, int, int]]]   # fwd[s]: transfers of forward boundary s (s -> s+1)
    bwd: List[List[Tuple[int, int, int]]]   # bwd[s]: transfers of backward boundary s (s+1 -> s)
    ar: List[int]                       # all-reduce duration per stage (0 if r_s = 1)


def stage_op_durations(f, b, a: int, e: int, ws: Sequence[int]) -> Tuple[dict, dict]:
    """Split replicas (reading C-3): F'_{s,w} = ceil(sum_{l=a..e} f[w][l] / r_s), same for B'.
    Table 1 rows FP_ij / BP_ij."""
    r = len(ws)
    Fd = {w: ceil_div(sum(f[w][a:e + 1]), r) for w in ws}
    Bd = {w: ceil_div(sum(b[w][a:e + 1]), r) for w in ws}
    return Fd, Bd


def allreduce_duration(P, a: int, e: int, ws: Sequence[int], tau) -> int:
    """Ring all-reduce of a replicated stage every mini-batch:
    2(r-1) steps of a ceil(P_s/r)-byte chunk over the slowest ring link, ring order = W_s ascending."""
    r = len(ws)
    if r < 2:
        return 0
    Ps = sum(P[a:e + 1])
    tau_ring = max(tau[ws[i]][ws[(i + 1) % r]] for i in range(r))
    return 2 * (r - 1) * xfer(ceil_div(Ps, r), tau_ring)


def ingredients(prof, st, part: Partition) -> Ingredients:
    L = len(prof.O)
    stages = part.stage_layers(L)
    Fd, Bd, ar = [], [], []
    for s, (a, e) in enumerate(stages):
        F_, B_ = stage_op_durations(st.f, st.b, a, e, part.W[s])
        Fd.append(F_)
        Bd.append(B_)
        ar.append(allreduce_duration(prof.P, a, e, part.W[s], st.tau))
    fwd, bwd = [], []
    for s in range(part.S - 1):
        e = stages[s][1]
        # forward: activation O[e_s] from W_s to W_{s+1}; backward: G[e_s+1] from W_{s+1} to W_s (C-6)
        fwd.append(boundary_transfers(prof.O[e], part.W[s], part.W[s + 1], st.tau))
        bwd.append(boundary_transfers(prof.G[e + 1], part.W[s + 1], part.W[s], st.tau))
    return Ingredients(part.S, part.W, Fd, Bd, fwd, bwd, ar)


def switch_bytes(prof, new: Partition, old: Partition) -> int:
    """SPEC §6: sum over layers l of P[l] * |W_new(l) minus W_old(l)| — the weights a worker must
    receive because it newly holds layer l (state switching moves layer weights)."""
    L = len(prof.O)

    def holders(p: Partition):
        h = [None] * L
        for s, (a, e) in enumerate(p.stage_layers(L)):
            for l in range(a, e + 1):
                h[l] = set(p.W[s])
        return h

    hn, ho = holders(new), holders(old)
    return sum(prof.P[l] * len(hn[l] - ho[l]) for l in range(L))
