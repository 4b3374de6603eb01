"""Oracle: the search space and its index order (SPEC.md §5). Test infrastructure only.

The paper enumerates candidate partitions and scores each with its speed model;
PipeDream solves the same space by DP "instead of exhaustive enumeration".
The order here is the definition: S ascending, then the worker composition R (a subset in
itertools.combinations order), then the cut set (also combinations order). Contiguous placement:
stage s gets workers [R_{s-1}, R_s) (reading C-11).
"""
from __future__ import annotations

from itertools import combinations
from math import comb
from typing import Iterator, List, Sequence, Tuple

from .model import Partition

USE_ALL_WORKERS = 1


def compositions(N: int, S: int, flags: int) -> Iterator[Tuple[int, ...]]:
    """Partial sums R_1 < ... < R_S in lexicographic order (sum r <= N, or = N with USE_ALL)."""
    if flags & USE_ALL_WORKERS:
        for head in combinations(range(1, N), S - 1):
            yield head + (N,)
    else:
        yield from combinations(range(1, N + 1), S)


def candidates(L: int, N: int, s_min: int, s_max: int, flags: int = 0) -> Iterator[Partition]:
    """Every candidate partition, in global index order (index = position in this iterator)."""
    for S in range(s_min, s_max + 1):
        for R in compositions(N, S, flags):
            W = [list(range(([0] + list(R))[s], R[s])) for s in range(S)]
            for cuts in combinations(range(L - 1), S - 1):
                yield Partition(S, list(cuts), [list(ws) for ws in W])


def count(L: int, N: int, s_min: int, s_max: int, flags: int = 0) -> int:
    total = 0
    for S in range(s_min, s_max + 1):
        k = comb(N - 1, S - 1) if flags & USE_ALL_WORKERS else comb(N, S)
        total += k * comb(L - 1, S - 1)
    return total


def lex_rank(subset: Sequence[int], n: int) -> int:
    """Position of a sorted k-subset of {0..n-1} in itertools.combinations order: the number of
    k-subsets that agree on a prefix and are smaller at the first position where they differ."""
    k = len(subset)
    rank, prev = 0, -1
    for i, c in enumerate(subset):
        for x in range(prev + 1, c):
            rank += comb(n - 1 - x, k - 1 - i)
        prev = c
    return rank


def lex_unrank(rank: int, n: int, k: int) -> List[int]:
    """Inverse of lex_rank: walk each position upward, skipping whole blocks of subsets."""
    out, x = [], 0
    for i in range(k):
        while comb(n - 1 - x, k - 1 - i) <= rank:
            rank -= comb(n - 1 - x, k - 1 - i)
            x += 1
        out.append(x)
        x += 1
    return out


def index_of(L: int, N: int, s_min: int, s_max: int, flags: int, part: Partition) -> int:
    """Global index of a contiguous candidate (SPEC §5)."""
    S = part.S
    off = count(L, N, s_min, S - 1, flags) if S > s_min else 0
    R = [ws[-1] + 1 for ws in part.W]
    if flags & USE_ALL_WORKERS:
        rho = lex_rank([x - 1 for x in R[:-1]], N - 1)
    else:
        rho = lex_rank([x - 1 for x in R], N)
    kappa = lex_rank(part.cuts, L - 1)
    return off + rho * comb(L - 1, S - 1) + kappa


def decode(L: int, N: int, s_min: int, s_max: int, flags: int, index: int) -> Partition:
    for S in range(s_min, s_max + 1):
        K = comb(N - 1, S - 1) if flags & USE_ALL_WORKERS else comb(N, S)
        block = K * comb(L - 1, S - 1)
        if index < block:
            rho, kappa = divmod(index, comb(L - 1, S - 1))
            if flags & USE_ALL_WORKERS:
                R = [x + 1 for x in lex_unrank(rho, N - 1, S - 1)] + [N]
            else:
                R = [x + 1 for x in lex_unrank(rho, N, S)]
            R0 = [0] + R
            W = [list(range(R0[s], R0[s + 1])) for s in range(S)]
            return Partition(S, lex_unrank(kappa, L - 1, S - 1), W)
        index -= block
    raise IndexError("index beyond the search space")
