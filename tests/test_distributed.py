"""Multi-process (world size 2, gloo, CPU) tests of the sharded search and the min-loc exchange.

The per-shard search is the oracle's brute force here (CPU); on the GPU it is the CUDA search of the
shard (tests/test_gpu_parity.py::test_gpt96_shards_match covers 8 shards on one device)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


class _OracleEngine:
    """Just the host-side support calls search_distributed needs (count, decode), from the oracle."""

    def __init__(self, L, N):
        self.L, self.N = L, N

    def count_candidates(self, s_min, s_max, flags):
        from oracle.enumerate import count
        return count(self.L, self.N, s_min, s_max, flags)

    def search_optimum_async(self, s_min, s_max, flags, begin, end):
        """The 40-byte autopipe_result of the oracle's brute force over the shard (a CPU tensor)."""
        import workloads as W
        from oracle.model import encode_partition
        from oracle.search import brute_force
        T, idx, part, n = brute_force(W.toy(), W.toy_state(), s_min, s_max, flags, begin=begin, end=end)
        if n == 0:
            T = idx = (1 << 64) - 1
        rec = encode_partition(part) if n else bytes([0xFF] * 16)
        raw = T.to_bytes(8, "little") + idx.to_bytes(8, "little") + n.to_bytes(8, "little") + rec
        return torch.frombuffer(bytearray(raw), dtype=torch.uint8).clone()

    def decode_index(self, s_min, s_max, flags, idx):
        from oracle.enumerate import decode
        from oracle.model import encode_partition
        return encode_partition(decode(self.L, self.N, s_min, s_max, flags, idx))


def _reduce_py(gathered):
    """Stand-in for autopipe_reduce_results on CPU: lexicographic (T, index) minimum, evaluated summed,
    the first minimal entry's record (its own definition, not the kernel's code)."""
    rows = [bytes(r.numpy().tobytes()) for r in gathered]
    key = lambda b: (int.from_bytes(b[0:8], "little"), int.from_bytes(b[8:16], "little"))
    best = min(range(len(rows)), key=lambda i: (key(rows[i]), i))
    total = sum(int.from_bytes(b[16:24], "little") for b in rows)
    out = rows[best][:16] + total.to_bytes(8, "little") + rows[best][24:]
    return torch.frombuffer(bytearray(out), dtype=torch.uint8).clone()


def _worker(rank, world, port, q, case):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import workloads as W
        from oracle.search import brute_force
        from paper_conf_icpp_hulww24_b200.distributed import minloc, search_distributed
        from paper_conf_icpp_hulww24_b200.engine import SearchResult
        if case == "minloc":
            vals = [(7, 30, 5), (7, 12, 9)] if world == 2 else [(7, 30, 5)]
            out = [minloc(*vals[rank])]
            # an empty shard on one rank
            out.append(minloc(*([(1 << 64) - 1, (1 << 64) - 1, 0], (3, 99, 4))[rank]))
            q.put((rank, out))
            return
        if case == "bound":  # the cross-shard bound's 8-byte exchange (uint64 in int64 storage)
            from paper_conf_icpp_hulww24_b200.distributed import bound_allreduce
            res = []
            for vals in ((416359965, 500000000), ((1 << 64) - 1, 480722219), ((1 << 64) - 1, (1 << 64) - 1)):
                t = torch.tensor([vals[rank] - (1 << 64) if vals[rank] >= (1 << 63) else vals[rank]],
                                 dtype=torch.int64)
                bound_allreduce(t)
                res.append(int(t.item()) & ((1 << 64) - 1))
            q.put((rank, res))
            return
        if case == "rollout":  # rollout batches: one slice per rank, outputs all-gathered (row e)
            from oracle.rollout import rollout_rewards
            from paper_conf_icpp_hulww24_b200.distributed import rollout_distributed
            prof, st = W.toy(), W.toy_state()
            recs = torch.from_numpy(W.sample_records(prof.L, st.N, 101, 7))
            cur = bytes(recs[3].numpy().tobytes())

            def score(sl, current):  # the oracle over the rank's slice (stand-in for the GPU call)
                ts, sws = rollout_rewards(prof, st, [bytes(r.numpy().tobytes()) for r in sl], current)
                to64 = lambda v: v - (1 << 64) if v >= (1 << 63) else v
                t = torch.tensor([to64(a) for a in ts], dtype=torch.int64)
                sw = torch.tensor([to64(b) for b in sws], dtype=torch.int64) if current is not None else None
                return t, sw
            t, sw = rollout_distributed(None, recs, cur, score=score)
            (lo, hi), t_own, _ = rollout_distributed(None, recs, None, score=score, gather=False)
            q.put((rank, ([int(x) & ((1 << 64) - 1) for x in t], [int(x) & ((1 << 64) - 1) for x in sw],
                          (lo, hi), [int(x) & ((1 << 64) - 1) for x in t_own])))
            return
        prof, st = W.toy(), W.toy_state()
        eng = _OracleEngine(prof.L, st.N)

        def shard(b, e):
            T, idx, part, n = brute_force(prof, st, 1, 4, 0, begin=b, end=e)
            if n == 0:
                return SearchResult((1 << 64) - 1, (1 << 64) - 1, 0, bytes([0xFF] * 16))
            return SearchResult(T, idx, n, b"")
        if case == "search_device":  # the default path: per-rank result bytes, gathered and reduced
            r = search_distributed(eng, 1, 4, 0, reduce_fn=_reduce_py)
        else:
            r = search_distributed(eng, 1, 4, 0, shard_search=shard)
        q.put((rank, (r.time_ns, r.index, r.evaluated, r.partition)))
    finally:
        dist.destroy_process_group()


def _run(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q, case)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=240) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def test_shard_bounds_cover_exactly():
    from paper_conf_icpp_hulww24_b200.distributed import shard_bounds
    for total in (0, 1, 7, 165, 11_050_084_695):
        for world in (1, 2, 3, 4, 8):
            prev = 0
            for r in range(world):
                lo, hi = shard_bounds(total, r, world)
                assert lo == prev and hi >= lo
                prev = hi
            assert prev == total


def test_minloc_gloo_world2():
    out = _run(2, "minloc")
    for rank in (0, 1):
        assert out[rank][0] == (7, 12, 14)          # tie on T: smaller index wins
        assert out[rank][1] == (3, 99, 4)           # an empty shard never wins


def test_search_distributed_gloo_world2_matches_single():
    from oracle.model import encode_partition
    from oracle.search import brute_force
    import workloads as W
    prof, st = W.toy(), W.toy_state()
    T, idx, part, n = brute_force(prof, st, 1, 4)
    out = _run(2, "search")
    for rank in (0, 1):
        assert out[rank] == (T, idx, n, encode_partition(part))


def test_search_distributed_device_minloc_gloo_world2():
    """The GPU path's exchange (all-gather of each rank's 40-byte result, then one reduction) with
    the shard searches and the reduction replaced by CPU stand-ins: same optimum, count and record as
    one process."""
    from oracle.model import encode_partition
    from oracle.search import brute_force
    import workloads as W
    prof, st = W.toy(), W.toy_state()
    T, idx, part, n = brute_force(prof, st, 1, 4)
    out = _run(2, "search_device")
    for rank in (0, 1):
        assert out[rank] == (T, idx, n, encode_partition(part))


def test_balanced_bounds_partition_the_space():
    """autopipe_balanced_shards (host-only): contiguous, ordered, covering exactly [0, total), for
    spaces with and without the fast kernel's blocks; G = 1 is the whole space."""
    from math import comb
    from oracle.enumerate import count
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    for (L, N, smin, smax, flags) in ((96, 8, 8, 8, 0), (96, 8, 1, 8, 0), (21, 8, 1, 8, 0), (8, 4, 1, 4, 0),
                                      (26, 8, 5, 8, 1), (18, 5, 1, 5, 1)):
        total = count(L, N, smin, smax, flags) if L < 60 else (
            comb(95, 7) if smin == 8 else sum(comb(N, S) * comb(L - 1, S - 1) for S in range(smin, smax + 1)))
        for G in (1, 2, 3, 8):
            b = balanced_bounds(L, N, smin, smax, flags, G)
            assert len(b) == G + 1 and b[0] == 0 and b[-1] == total
            assert all(x <= y for x, y in zip(b, b[1:]))
    # wide spaces (row f4): 10 and 16 workers, stages beyond 8
    for (L, N, smin, smax, flags) in ((12, 10, 1, 10, 0), (20, 16, 9, 12, 1), (30, 12, 5, 12, 0)):
        total = count(L, N, smin, smax, flags)
        for G in (1, 3, 8):
            b = balanced_bounds(L, N, smin, smax, flags, G)
            assert len(b) == G + 1 and b[0] == 0 and b[-1] == total
            assert all(x <= y for x, y in zip(b, b[1:]))
    # the 96-layer space: later shards (short rows) get fewer candidates than earlier ones
    b = balanced_bounds(96, 8, 8, 8, 0, 8)
    sizes = [y - x for x, y in zip(b, b[1:])]
    assert sizes[-1] < sizes[0] and abs(sum(sizes) - comb(95, 7)) == 0
    # per integer path (autopipe_balanced_shards_path): the 64-bit model is the default one; the
    # 32-bit model weighs rows more, so its interior bounds move toward the end of the space
    assert balanced_bounds(96, 8, 8, 8, 0, 8, 64) == b
    b32 = balanced_bounds(96, 8, 8, 8, 0, 8, 32)
    assert b32[0] == 0 and b32[-1] == comb(95, 7) and all(x <= y for x, y in zip(b32, b32[1:]))
    assert all(x >= y for x, y in zip(b32[1:-1], b[1:-1]))
    for (L, N, smin, smax, flags) in ((21, 8, 1, 8, 0), (26, 8, 5, 8, 1)):
        total = count(L, N, smin, smax, flags)
        for G in (1, 3, 8):
            b = balanced_bounds(L, N, smin, smax, flags, G, 32)
            assert len(b) == G + 1 and b[0] == 0 and b[-1] == total
            assert all(x <= y for x, y in zip(b, b[1:]))


def test_balanced_bounds_rejects_bad_arguments():
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    for args in ((96, 8, 0, 8, 0, 2), (96, 8, 3, 2, 0, 2), (96, 4, 1, 5, 0, 2), (96, 8, 1, 8, 2, 2),
                 (96, 8, 1, 8, 0, 0), (0, 8, 1, 1, 0, 1), (256, 8, 1, 8, 0, 1), (96, 17, 1, 8, 0, 2),
                 (96, 16, 1, 17, 0, 2)):
        with pytest.raises(ValueError):
            balanced_bounds(*args)
    import ctypes
    from paper_conf_icpp_hulww24_b200._lib import lib
    out = (ctypes.c_uint64 * 3)()
    assert lib.autopipe_balanced_shards_path(96, 8, 8, 8, 0, 2, 16, out) != 0  # int_path must be 32 or 64


def test_bound_allreduce_gloo_world2():
    """Row e, cross-shard bound: the ranks' seed words min-reduced as uint64 (UINT64_MAX = no seed
    never wins over a real seed, and stays UINT64_MAX when no rank has one)."""
    out = _run(2, "bound")
    for rank in (0, 1):
        assert out[rank] == [416359965, 480722219, (1 << 64) - 1]


@pytest.mark.parametrize("world", [2, 3])
def test_rollout_distributed_gloo(world):
    """Row e for rollout batches: 101 records split over 2 or 3 ranks (uneven slices, padded for the
    all-gather), every rank ends with the whole batch's (T, switch bytes) = the oracle's, in order."""
    import workloads as W
    from oracle.rollout import rollout_rewards
    from paper_conf_icpp_hulww24_b200.distributed import shard_bounds
    prof, st = W.toy(), W.toy_state()
    recs = W.sample_records(prof.L, st.N, 101, 7)
    cur = bytes(recs[3])
    want = list(zip(*rollout_rewards(prof, st, [bytes(r) for r in recs], cur)))
    out = _run(world, "rollout")
    for rank in range(world):
        t, sw, (lo, hi), t_own = out[rank]
        assert t == [a for a, _ in want] and sw == [b for _, b in want]
        assert (lo, hi) == shard_bounds(101, rank, world)
        assert t_own == [a for a, _ in want[lo:hi]]
