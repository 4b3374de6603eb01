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

constexpr u32 RR_SIM_ROUNDS = 4096;         // then ceil(lambda) from the event graph (rr_ceil_bf)
constexpr int RR_BF_NODES = 160;            // 4 S Lam <= 144 nodes for sum r <= 8
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

// ceil(lambda_compute) from the timed event graph of one period (the oracle's event_graph): the
// smallest integer theta with no positive cycle of node durations - theta * Lam * edge tokens
// (Bellman-Ford from a virtual source, binary search on theta, bracketed around the simulation's
// estimate th0). Nodes (kind, s, phase p): F_s, B_s, forward and backward transfers of boundary s, for
// the mini-batches k = p (mod Lam). For the rare records whose simulation has not settled (two
// near-equal cycle ratios can make the transient arbitrarily long); exact like the simulation.
template <typename DurF>
__device__ __forceinline__ u64 rr_ceil_bf(int S, u32 Lam, const int *r, const int *m, const int *lc, DurF dur,
                                          long long th0) {
  const int V = 4 * S * (int)Lam;
  long long dist[RR_BF_NODES];
  const long long K0 = 64ll * Lam;  // a period index far from the start: every predecessor is >= 0
  auto node = [&](int kind, int s, long long k) { return (kind * S + s) * (int)Lam + (int)(k % Lam); };
  auto tok = [&](long long kv, long long ku) { return kv / (long long)Lam - ku / (long long)Lam; };
  auto positive = [&](long long th) -> bool {
    for (int v = 0; v < V; ++v) dist[v] = 0;
    for (int pass = 0; pass <= V; ++pass) {
      bool changed = false;
      for (int kind = 0; kind < 4; ++kind)
        for (int s = 0; s < S; ++s) {
          if (kind >= 2 && s == S - 1) continue;
          for (u32 p = 0; p < Lam; ++p) {
            const long long k = K0 + p;
            const int v = node(kind, s, k);
            const long long dv = (long long)dur(kind, s, (int)p);
            long long best = dist[v];
            auto relax = [&](int ku_kind, int ku_s, long long ku) {
              const long long c = dist[node(ku_kind, ku_s, ku)] + dv - th * (long long)Lam * tok(k, ku);
              if (c > best) best = c;
            };
            if (kind == 0) {
              relax(1, s, k - (long long)m[s] * r[s]);         // worker order: after B(k - m r)
              if (s > 0) relax(2, s - 1, k);                   // forward transfer of boundary s-1
            } else if (kind == 1) {
              relax(0, s, k + (long long)(m[s] - 1) * r[s]);   // worker order: after F(k + (m-1) r)
              if (s < S - 1) relax(3, s, k);                   // backward transfer of boundary s
            } else if (kind == 2) {
              relax(0, s, k);                                  // after F_s(k)
              relax(2, s, k - lc[s]);                          // FIFO on its link
            } else {
              relax(1, s + 1, k);                              // after B_{s+1}(k)
              relax(3, s, k - lc[s]);
            }
            if (best > dist[v]) {
              dist[v] = best;
              changed = true;
            }
          }
        }
      if (!changed) return false;
    }
    return true;
  };
  // bracket [lo, hi]: positive(lo), !positive(hi), around the estimate
  long long lo, hi, step = 1;
  if (positive(th0)) {
    lo = th0;
    hi = th0 + step;
    while (positive(hi)) lo = hi, step *= 2, hi = th0 + step;
  } else {
    hi = th0;
    lo = th0 - step;
    while (lo >= 0 && !positive(lo)) hi = lo, step *= 2, lo = th0 - step;
    if (lo < 0) lo = -1;
  }
  while (hi - lo > 1) {
    const long long mid = lo + (hi - lo) / 2;
    if (positive(mid)) lo = mid;
    else hi = mid;
  }
  return (u64)hi;
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
  // phases of the next op of every stage (mini-batch mod r_s, mod lcm of its boundary), advanced by
  // one per round once the stage's mini-batch index is >= 0 (no 64-bit modulo in the recurrence)
  int bph[MAXS], bl[MAXS], fph[MAXS], fl[MAXS];
  for (int s = 0; s < S; ++s) bph[s] = bl[s] = fph[s] = fl[s] = 0;
  auto step = [](int &ph, int m) { ph = (ph + 1 == m) ? 0 : ph + 1; };
  auto round = [&]() {
    u64 bd = 0;
    if (j >= 0) {
      for (int s = S - 1; s >= 0; --s) {  // B_s(j), backward boundary s-1 of mini-batch j
        const int w = (wl[s] >> (4 * bph[s])) & 15;
        step(bph[s], r[s]);
        const u64 end = umax(wf[w], s == S - 1 ? 0ull : bd) + Bw[w];
        wf[w] = end;
        if (s > 0) {
          const int q = lo[s - 1] + bl[s];
          step(bl[s], lc[s - 1]);
          const u64 fin = umax(end, lfb[q]) + tb[q];
          lfb[q] = fin;
          bd = fin;
        }
      }
    }
    for (int s = 0; s < S; ++s) {  // F_s(j + D_s), forward boundary s of that mini-batch
      const long long k = j + D[s];
      if (k < 0) continue;
      const int w = (wl[s] >> (4 * fph[s])) & 15;
      step(fph[s], r[s]);
      const u64 end = umax(wf[w], s == 0 ? 0ull : fdr[s - 1][k & (RR_RING - 1)]) + Fw[w];
      wf[w] = end;
      if (s < S - 1) {
        const int q = lo[s] + fl[s];
        step(fl[s], lc[s]);
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
    for (int s = 0; s < S - 1; ++s)  // pending forward transfers in logical order (from j + D_{s+1})
      for (int q = 0; q < D[s] - D[s + 1]; ++q) {
        const long long k = j + D[s + 1] + q;
        tfd[s][q] = k >= 0 ? fdr[s][k & (RR_RING - 1)] : U64MAX;
      }
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
      for (int q = 0; q < D[s] - D[s + 1]; ++q) {
        const long long k = j + D[s + 1] + q;
        if ((k >= 0 ? fdr[s][k & (RR_RING - 1)] : U64MAX) != tfd[s][q]) return false;
      }
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
  bool settled = true;
  while (!same()) {
    if (power == lam) {
      save();
      power *= 2;
      lam = 0;
    }
    block();
    ++lam;
    rounds += Lam;
    if (rounds > RR_SIM_ROUNDS) {
      settled = false;
      break;
    }
  }
  const u64 den = (u64)lam * Lam;
  u64 T = 0;
  for (u32 c = 0; c < g; ++c) T = umax(T, (off[c] + den - 1) / den);
  if (!settled) {
    int mm[MAXS];
    {
      int R = 0;
      for (int s = S - 1; s >= 0; --s) R += r[s], mm[s] = (R + r[s] - 1) / r[s];
    }
    auto dur = [&](int kind, int s, int ph) -> u64 {
      if (kind <= 1) {
        const int w = (wl[s] >> (4 * (ph % r[s]))) & 15;
        return kind == 0 ? Fw[w] : Bw[w];
      }
      const int q = lo[s] + ph % lc[s];
      return kind == 2 ? tf[q] : tb[q];
    };
    T = rr_ceil_bf(S, Lam, r, mm, lc, dur, (long long)T);
  }
  return umax(T, Tsync);
}

}  // namespace ap
