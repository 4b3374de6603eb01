// rr.cuh — NEXT row f4: PipeDream's round-robin replicas (reading F-5; oracle/roundrobin.py).
//
// A replicated stage takes whole mini-batches in turn: mini-batch k runs at stage s on replica
// k mod r_s with its full F and B (PipeDream picks the stages, the "number of
// workers for each stage" and the "number of on-the-fly mini-batches"). Replica i runs 1F1B over its
// own mini-batches with m_s = ceil(R_s / r_s) in flight (R_s = workers of stages s..S-1; NOAM for the
// input stage); boundary s of mini-batch k is one transfer on W_s[k mod r_s] -> W_{s+1}[k mod r_{s+1}]
// (forward O[e_s]) and back (G[e_s + 1]), FIFO per directed link; a replicated stage synchronises
// once per r_s mini-batches, overlapped: T = max(ceil(lambda_compute), max_s ceil(d_s / r_s)).
//
// lambda_compute has no closed form here; one thread finds it exactly by running the schedule's
// max-plus recurrence round by round in dependency order (round j: B_s(j) for s descending, then
// F_s(j + D_s) for s ascending, D_s = min_{u<=s} m_u r_u; every op's inputs are produced earlier)
// and detecting the periodic regime with Brent's cycle search over the state at the start of
// every block of Lam = lcm(r) rounds: the free time of every worker and link and the forward
// transfers not yet consumed, rebased per class of mini-batches (k mod gcd(r): classes share no
// worker and no link). When the rebased state repeats after c blocks, each class has advanced by
// its shift D_c: lambda_compute = max_c D_c / (c Lam). The oracle finds the same period by hashing
// windows of rounds in a generic ready-driven simulation.
#pragma once
#include "eval.cuh"

namespace ap {

constexpr u64 RR_UNRESOLVED = U64MAX - 1;   // no periodic regime within RR_MAX_ROUNDS (both sides)
constexpr u32 RR_MAX_ROUNDS = 1u << 18;
constexpr int RR_LINKS = 32;                // sum over boundaries of lcm(r_s, r_{s+1}) for N <= 8
constexpr int RR_RING = 16;                 // pending forward transfers per boundary (D_0 <= 15)

__device__ __forceinline__ u32 gcd_u(u32 a, u32 b) {
  while (b) {
    const u32 t = a % b;
    a = b;
    b = t;
  }
  return a;
}

// T_ns of a validated 16-byte partition under round-robin replicas.
static __device__ __noinline__ u64 rr_time(const SmemTab &t, int S, const P8 &p, int sync) {
  int r[MAXS], wl[MAXS], D[MAXS], lc[MAXS], lo[MAXS];
  u64 Fw[MAXN], Bw[MAXN];
  u64 Tsync = 0;
  u32 Lam = 1, g = 0;
  for (int s = 0; s < S; ++s) {
    const u32 mask = p.mask(s);
    r[s] = __popc(mask);
    const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
    const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
    int packed = 0, i = 0;
    for (u32 mm = mask; mm; mm &= mm - 1, ++i) {
      const int w = __ffs(mm) - 1;
      packed |= w << (4 * i);
      Fw[w] = t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a];  // whole mini-batch: no split
      Bw[w] = t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a];
    }
    wl[s] = packed;
    if (r[s] >= 2) {  // one synchronisation per r_s mini-batches
      const u64 d = sync_time<8>(sync, t.PP[e + 1] - t.PP[a], mask, t.tau, t.dv);
      Tsync = umax(Tsync, (d + r[s] - 1) / (u64)r[s]);
    }
    Lam = Lam / gcd_u(Lam, (u32)r[s]) * (u32)r[s];
    g = gcd_u(g, (u32)r[s]);
  }
  if (S == 1) {  // no boundary: each replica on its own, one mini-batch in every r
    u64 T = 0;
    for (int i = 0; i < r[0]; ++i) {
      const int w = (wl[0] >> (4 * i)) & 15;
      T = umax(T, (Fw[w] + Bw[w] + r[0] - 1) / (u64)r[0]);
    }
    return umax(T, Tsync);
  }
  // in flight per replica, forward round offsets, link slots (one per phase k mod lcm(r_s, r_{s+1}))
  u64 tf[RR_LINKS], tb[RR_LINKS];
  {
    int R = 0;
    for (int s = S - 1; s >= 0; --s) R += r[s], D[s] = ((R + r[s] - 1) / r[s]) * r[s];
    for (int s = 1; s < S; ++s) D[s] = D[s] < D[s - 1] ? D[s] : D[s - 1];
    int off = 0;
    for (int s = 0; s < S - 1; ++s) {
      lc[s] = r[s] / (int)gcd_u((u32)r[s], (u32)r[s + 1]) * r[s + 1];
      lo[s] = off;
      const int eb = p.cut(s);
      for (int k = 0; k < lc[s]; ++k) {
        const int u = (wl[s] >> (4 * (k % r[s]))) & 15, v = (wl[s + 1] >> (4 * (k % r[s + 1]))) & 15;
        tf[off + k] = xfer(t.O[eb], t.tau[u * TAUW + v]);
        tb[off + k] = xfer(t.G[eb + 1], t.tau[v * TAUW + u]);
      }
      off += lc[s];
    }
  }
  // schedule state
  u64 wf[MAXN], lff[RR_LINKS], lfb[RR_LINKS], fdr[MAXS - 1][RR_RING];
  for (int w = 0; w < MAXN; ++w) wf[w] = 0;
  for (int q = 0; q < RR_LINKS; ++q) lff[q] = lfb[q] = 0;
  long long j = -(long long)D[0];  // the first round with an op: F_0(0)
  auto round = [&]() {
    u64 bd = 0;
    if (j >= 0) {
      for (int s = S - 1; s >= 0; --s) {  // B_s(j), backward boundary s-1 of mini-batch j
        const int w = (wl[s] >> (4 * (int)(j % r[s]))) & 15;
        const u64 end = umax(wf[w], s == S - 1 ? 0ull : bd) + Bw[w];
        wf[w] = end;
        if (s > 0) {
          const int q = lo[s - 1] + (int)(j % lc[s - 1]);
          const u64 fin = umax(end, lfb[q]) + tb[q];
          lfb[q] = fin;
          bd = fin;
        }
      }
    }
    for (int s = 0; s < S; ++s) {  // F_s(j + D_s), forward boundary s of that mini-batch
      const long long k = j + D[s];
      if (k < 0) continue;
      const int w = (wl[s] >> (4 * (int)(k % r[s]))) & 15;
      const u64 end = umax(wf[w], s == 0 ? 0ull : fdr[s - 1][k & (RR_RING - 1)]) + Fw[w];
      wf[w] = end;
      if (s < S - 1) {
        const int q = lo[s] + (int)(k % lc[s]);
        const u64 fin = umax(end, lff[q]) + tf[q];
        lff[q] = fin;
        fdr[s][k & (RR_RING - 1)] = fin;
      }
    }
    ++j;
  };
  // the live state at a block boundary (j = the next round): per class c = k mod g, its minimum is
  // subtracted (rebase) and added to off[c]
  u64 off[MAXN], tw[MAXN], tlf[RR_LINKS], tlb[RR_LINKS], tfd[MAXS - 1][RR_RING];
  auto rebase = [&]() {
    u64 mn[MAXN];
    for (u32 c = 0; c < g; ++c) mn[c] = U64MAX;
    for (int s = 0; s < S; ++s)
      for (int i = 0; i < r[s]; ++i) {
        const int w = (wl[s] >> (4 * i)) & 15;
        mn[i % g] = umin(mn[i % g], wf[w]);
      }
    for (int s = 0; s < S - 1; ++s)
      for (int k = 0; k < lc[s]; ++k) {
        mn[k % g] = umin(mn[k % g], umin(lff[lo[s] + k], lfb[lo[s] + k]));
      }
    for (int s = 0; s < S - 1; ++s)  // pending forward transfers of boundary s: k in (j-1+D_{s+1}, j-1+D_s]
      for (long long k = j + D[s + 1]; k < j + D[s]; ++k)
        if (k >= 0) mn[(u32)(k % g)] = umin(mn[(u32)(k % g)], fdr[s][k & (RR_RING - 1)]);
    for (u32 c = 0; c < g; ++c) off[c] += mn[c];
    for (int s = 0; s < S; ++s)
      for (int i = 0; i < r[s]; ++i) {
        const int w = (wl[s] >> (4 * i)) & 15;
        wf[w] -= mn[i % g];
      }
    for (int s = 0; s < S - 1; ++s)
      for (int k = 0; k < lc[s]; ++k) {
        lff[lo[s] + k] -= mn[k % g];
        lfb[lo[s] + k] -= mn[k % g];
      }
    for (int s = 0; s < S - 1; ++s)
      for (long long k = j + D[s + 1]; k < j + D[s]; ++k)
        if (k >= 0) fdr[s][k & (RR_RING - 1)] -= mn[(u32)(k % g)];
  };
  auto save = [&]() {
    for (int w = 0; w < MAXN; ++w) tw[w] = wf[w];
    for (int q = 0; q < RR_LINKS; ++q) tlf[q] = lff[q], tlb[q] = lfb[q];
    for (int s = 0; s < S - 1; ++s)
      for (int q = 0; q < RR_RING; ++q) tfd[s][q] = fdr[s][q];
    for (u32 c = 0; c < g; ++c) off[c] = 0;
  };
  auto same = [&]() -> bool {
    for (int s = 0; s < S; ++s)
      for (int i = 0; i < r[s]; ++i) {
        const int w = (wl[s] >> (4 * i)) & 15;
        if (wf[w] != tw[w]) return false;
      }
    for (int s = 0; s < S - 1; ++s)
      for (int k = 0; k < lc[s]; ++k)
        if (lff[lo[s] + k] != tlf[lo[s] + k] || lfb[lo[s] + k] != tlb[lo[s] + k]) return false;
    for (int s = 0; s < S - 1; ++s)
      for (long long k = j + D[s + 1]; k < j + D[s]; ++k)
        if (k >= 0 && fdr[s][k & (RR_RING - 1)] != tfd[s][k & (RR_RING - 1)]) return false;
    return true;
  };
  auto block = [&]() {
    for (u32 q = 0; q < Lam; ++q) round();
    rebase();
  };
  for (u32 c = 0; c < MAXN; ++c) off[c] = 0;
  // Brent: the tortoise jumps to the hare at powers of two; lam = blocks since the tortoise
  block();
  save();
  block();
  u32 power = 1, lam = 1, rounds = 2 * Lam;
  while (!same()) {
    if (power == lam) {
      save();
      power *= 2;
      lam = 0;
    }
    block();
    ++lam;
    rounds += Lam;
    if (rounds > RR_MAX_ROUNDS) return RR_UNRESOLVED;
  }
  const u64 den = (u64)lam * Lam;
  u64 T = 0;
  for (u32 c = 0; c < g; ++c) T = umax(T, (off[c] + den - 1) / den);
  return umax(T, Tsync);
}

}  // namespace ap
