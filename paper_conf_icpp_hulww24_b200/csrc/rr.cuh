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
// lambda_compute has no closed form here. One thread runs the schedule's max-plus recurrence round
// by round in dependency order (round j: B_s(j) for s descending, then F_s(j + D_s) for s ascending,
// D_s = min_{u<=s} m_u r_u; every op's inputs are produced earlier), one block of Lam = lcm(r)
// rounds at a time, and compares the state (the free time of every worker and link and the forward
// transfers not yet consumed) with a saved one (Brent's tortoise): per class of mini-batches
// (k mod gcd(r): classes share no worker and no link) the growth of every component since the save
// bounds that class's rate from both sides (max-plus homogeneity), and T is exact as soon as the
// ceilings of the two bounds agree — in particular when the schedule has repeated (every component
// of a class moved by the same amount). The oracle finds the period by hashing windows of rounds in
// a generic ready-driven simulation.
//
// Records whose bounds have not met within a round budget (two near-equal cycle ratios can make the
// transient arbitrarily long) take ceil(lambda) from the timed event graph of one period: the
// smallest integer theta with no positive cycle (Bellman-Ford, binary search on theta inside the
// bracket the bounds give). The eval kernel defers them to a drain kernel that runs the
// Bellman-Ford passes with a whole warp per record (k_eval.cu), so one slow record does not hold up
// the 31 other lanes of its warp; the search kernels run it in the thread.
#pragma once
#include <climits>
#include <cmath>

#include "eval.cuh"

namespace ap {

#ifndef RR_STATS
#define RR_STATS 0
#endif
constexpr u32 RR_SIM_ROUNDS = 4096;    // in-thread budget when nothing is deferred (AUTOPIPE_RR_NO_DEFER)
constexpr int RR_BF_NODES = 160;       // 4 S Lam <= 144 nodes for sum r <= 8
constexpr int RR_LINKS = 16;           // max over sum r <= 8 of sum_s lcm(r_s, r_{s+1}) (r = 1, 4, 3)
constexpr int RR_PEND = 24;            // pending forward transfers: sum_s (D_s - D_{s+1} + 1) <= 15 + 7

__device__ __forceinline__ u32 gcd_u(u32 a, u32 b) {
  while (b) {
    const u32 t = a % b;
    a = b;
    b = t;
  }
  return a;
}

// Everything the recurrence and the event graph need about one validated 16-byte record.
struct RRSetup {
  int S;
  u32 Lam, g;   // lcm and gcd of the replica counts
  u64 Tsync;    // max_s ceil(sync_s / r_s) over the replicated stages
  u64 dsum;     // sum of every op and transfer duration of one period
  int negtok;   // the most negative token count of an edge, negated (B_s(k) after F_s(k + (m - 1) r))
  int r[MAXS], wl[MAXS], D[MAXS], mm[MAXS], lc[MAXS], lo[MAXS];
  u64 Fw[MAXN], Bw[MAXN], tf[RR_LINKS], tb[RR_LINKS];
};

__device__ __forceinline__ void rr_setup(const SmemTab &t, int S, const P8 &p, int sync, RRSetup &R) {
  R.S = S;
  R.Tsync = 0;
  R.Lam = 1;
  R.g = 0;
  for (int s = 0; s < S; ++s) {
    const u32 mask = p.mask(s);
    R.r[s] = __popc(mask);
    const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
    const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
    int packed = 0, i = 0;
    for (u32 mm = mask; mm; mm &= mm - 1, ++i) {
      const int w = __ffs(mm) - 1;
      packed |= w << (4 * i);
      R.Fw[w] = t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a];  // whole mini-batch: no split
      R.Bw[w] = t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a];
    }
    R.wl[s] = packed;
    if (R.r[s] >= 2) {  // one synchronisation per r_s mini-batches
      const u64 d = sync_time<8>(sync, t.PP[e + 1] - t.PP[a], mask, t.tau, t.dv);
      R.Tsync = umax(R.Tsync, (d + R.r[s] - 1) / (u64)R.r[s]);
    }
    R.Lam = R.Lam / gcd_u(R.Lam, (u32)R.r[s]) * (u32)R.r[s];
    R.g = gcd_u(R.g, (u32)R.r[s]);
  }
  // in flight per replica, forward round offsets, link slots (one per phase k mod lcm(r_s, r_{s+1}))
  int Rs = 0;
  for (int s = S - 1; s >= 0; --s) {
    Rs += R.r[s];
    R.mm[s] = (Rs + R.r[s] - 1) / R.r[s];
    R.D[s] = R.mm[s] * R.r[s];
  }
  for (int s = 1; s < S; ++s) R.D[s] = R.D[s] < R.D[s - 1] ? R.D[s] : R.D[s - 1];
  R.negtok = 0;
  for (int s = 0; s < S; ++s) {
    const int nt = ((R.mm[s] - 1) * R.r[s]) / (int)R.Lam + 1;
    R.negtok = nt > R.negtok ? nt : R.negtok;
  }
  u64 dsum = 0;
  for (int s = 0; s < S; ++s)
    for (int i = 0; i < R.r[s]; ++i) {
      const int w = (R.wl[s] >> (4 * i)) & 15;
      dsum += (R.Fw[w] + R.Bw[w]) * (R.Lam / (u32)R.r[s]);
    }
  int off = 0;
  for (int s = 0; s < S - 1; ++s) {
    R.lc[s] = R.r[s] / (int)gcd_u((u32)R.r[s], (u32)R.r[s + 1]) * R.r[s + 1];
    R.lo[s] = off;
    const int eb = p.cut(s);
    for (int k = 0; k < R.lc[s]; ++k) {
      const int u = (R.wl[s] >> (4 * (k % R.r[s]))) & 15, v = (R.wl[s + 1] >> (4 * (k % R.r[s + 1]))) & 15;
      R.tf[off + k] = xfer(t.O[eb], t.tau[u * TAUW + v]);
      R.tb[off + k] = xfer(t.G[eb + 1], t.tau[v * TAUW + u]);
      dsum += (R.tf[off + k] + R.tb[off + k]) * (R.Lam / (u32)R.lc[s]);
    }
    off += R.lc[s];
  }
  R.dsum = dsum;
}

// S = 1: no boundary; each replica runs F, B, F, B, ... on its own mini-batches (one in every r)
__device__ __forceinline__ u64 rr_single_stage(const RRSetup &R) {
  u64 T = 0;
  for (int i = 0; i < R.r[0]; ++i) {
    const int w = (R.wl[0] >> (4 * i)) & 15;
    T = umax(T, (R.Fw[w] + R.Bw[w] + R.r[0] - 1) / (u64)R.r[0]);
  }
  return T;
}

// A lower bound on ceil(lambda_compute) from single-resource cycles: a replica of stage s runs F + B
// of one in every r_s mini-batches, a link slot of boundary s carries one in every lcm(r_s, r_{s+1}).
__device__ __forceinline__ u64 rr_lower(const RRSetup &R) {
  u64 lb = 0;
  for (int s = 0; s < R.S; ++s)
    for (int i = 0; i < R.r[s]; ++i) {
      const int w = (R.wl[s] >> (4 * i)) & 15;
      lb = umax(lb, (R.Fw[w] + R.Bw[w] + R.r[s] - 1) / (u64)R.r[s]);
    }
  for (int s = 0; s < R.S - 1; ++s)
    for (int k = 0; k < R.lc[s]; ++k) {
      const int q = R.lo[s] + k;
      lb = umax(lb, (umax(R.tf[q], R.tb[q]) + R.lc[s] - 1) / (u64)R.lc[s]);
    }
  return lb;
}

enum { RR_MET = 0, RR_BUDGET = 1, RR_PRUNED = 2, RR_CONT = 3 };
// The recurrence as a resumable state machine (S >= 2): init() runs the warm-up blocks (until every
// stage has started, j >= 0) and saves the tortoise; each step() runs one block of Lam rounds and
// decides: RR_MET: t_lo = t_hi = ceil(lambda_compute), the growth bounds met; RR_PRUNED: t_lo > prune
// (a search candidate that cannot win); RR_BUDGET: more than `cap` rounds, t_lo <= ceil(lambda_compute)
// <= t_hi; RR_CONT: not decided yet. (Resuming it block by block to refill decided lanes with the
// warp's next records was measured no faster: DESIGN.md §10.)
struct RRSim {
  // absolute times (no rebasing: < 2^58 within the round cap for a state bound below 2^45, checked by
  // the host)
  // forward transfers not yet consumed: boundary s keeps a FIFO of D_s - D_{s+1} + 1 slots at
  // fo[s] in fdr (F_s(k) writes the slot F_{s+1}(k) reads D_s - D_{s+1} rounds later; the extra slot
  // lets the write of round j precede that round's read), write / read positions fw[s] / fr[s]
  u64 wf[MAXN], lff[RR_LINKS], lfb[RR_LINKS], fdr[RR_PEND];
  // the saved state (Brent's tortoise): worker and link free times and the pending forward
  // transfers in logical order (mini-batch j + D_{s+1} + q, boundary s at fo[s])
  u64 tw[MAXN], tlf[RR_LINKS], tlb[RR_LINKS], tfd[RR_PEND];
  int fo[MAXS], fw[MAXS], fr[MAXS];
  long long j;  // the next round
  // phases of the next op of every stage (mini-batch mod r_s, mod lcm of its boundary), advanced by
  // one per round once the stage's mini-batch index is >= 0 (no 64-bit modulo in the recurrence)
  int bph[MAXS], bl[MAXS], fph[MAXS], fl[MAXS];
  u32 rounds, power, lam;

  // one block = Lam rounds; round j: B_s(j) for s descending (with the backward transfer of boundary
  // s - 1), then F_s(j + D_s) for s ascending (with the forward transfer of boundary s)
  __device__ __forceinline__ void block(const RRSetup &R) {
    const int S = R.S;
    for (u32 q = 0; q < R.Lam; ++q, ++j) {
      u64 bd = 0;
      if (j >= 0) {
        for (int s = S - 1; s >= 0; --s) {
          const int w = (R.wl[s] >> (4 * bph[s])) & 15;
          bph[s] = bph[s] + 1 == R.r[s] ? 0 : bph[s] + 1;
          const u64 end = umax(wf[w], bd) + R.Bw[w];
          wf[w] = end;
          if (s > 0) {
            const int ql = R.lo[s - 1] + bl[s];
            bl[s] = bl[s] + 1 == R.lc[s - 1] ? 0 : bl[s] + 1;
            bd = umax(end, lfb[ql]) + R.tb[ql];
            lfb[ql] = bd;
          }
        }
      }
      for (int s = 0; s < S; ++s) {
        const long long k = j + R.D[s];
        if (k < 0) continue;
        const int w = (R.wl[s] >> (4 * fph[s])) & 15;
        fph[s] = fph[s] + 1 == R.r[s] ? 0 : fph[s] + 1;
        u64 in = 0;
        if (s > 0) {
          const int len = R.D[s - 1] - R.D[s] + 1;
          in = fdr[fo[s - 1] + fr[s - 1]];
          fr[s - 1] = fr[s - 1] + 1 == len ? 0 : fr[s - 1] + 1;
        }
        const u64 end = umax(wf[w], in) + R.Fw[w];
        wf[w] = end;
        if (s < S - 1) {
          const int ql = R.lo[s] + fl[s];
          fl[s] = fl[s] + 1 == R.lc[s] ? 0 : fl[s] + 1;
          const u64 fd = umax(end, lff[ql]) + R.tf[ql];
          lff[ql] = fd;
          const int len = R.D[s] - R.D[s + 1] + 1;
          fdr[fo[s] + fw[s]] = fd;
          fw[s] = fw[s] + 1 == len ? 0 : fw[s] + 1;
        }
      }
    }
  }
  __device__ __forceinline__ void save(const RRSetup &R) {
    for (int w = 0; w < MAXN; ++w) tw[w] = wf[w];
    for (int q = 0; q < RR_LINKS; ++q) tlf[q] = lff[q], tlb[q] = lfb[q];
    for (int s = 0; s < R.S - 1; ++s) {
      const int len = R.D[s] - R.D[s + 1] + 1;
      for (int q = 0, x = fr[s]; q < len - 1; ++q, x = x + 1 == len ? 0 : x + 1) tfd[fo[s] + q] = fdr[fo[s] + x];
    }
  }
  // Growth since the save, lam blocks ago (max-plus): the block map is monotone and additively
  // homogeneous per class, so if every live component of class c moved by delta_i, class c's rate
  // lies in [min delta_i, max delta_i] per lam blocks; lambda = max_c rate_c.
  __device__ __forceinline__ void bounds(const RRSetup &R, u64 den, u64 &t_lo, u64 &t_hi) const {
    const int S = R.S;
    const u32 g = R.g;
    long long mn[MAXN], mx[MAXN];
    for (u32 c = 0; c < g; ++c) mn[c] = LLONG_MAX, mx[c] = LLONG_MIN;
    for (int s = 0; s < S; ++s)
      for (int i = 0; i < R.r[s]; ++i) {
        const int w = (R.wl[s] >> (4 * i)) & 15;
        const long long d = (long long)(wf[w] - tw[w]);
        const u32 c = (u32)i % g;
        mn[c] = d < mn[c] ? d : mn[c];
        mx[c] = d > mx[c] ? d : mx[c];
      }
    for (int s = 0; s < S - 1; ++s)
      for (int k = 0; k < R.lc[s]; ++k) {
        const int ql = R.lo[s] + k;
        const long long d1 = (long long)(lff[ql] - tlf[ql]), d2 = (long long)(lfb[ql] - tlb[ql]);
        const u32 c = (u32)k % g;
        mn[c] = d1 < mn[c] ? d1 : mn[c];
        mx[c] = d1 > mx[c] ? d1 : mx[c];
        mn[c] = d2 < mn[c] ? d2 : mn[c];
        mx[c] = d2 > mx[c] ? d2 : mx[c];
      }
    for (int s = 0; s < S - 1; ++s) {
      const int len = R.D[s] - R.D[s + 1] + 1;
      for (int q = 0, x = fr[s]; q < len - 1; ++q, x = x + 1 == len ? 0 : x + 1) {
        const long long k = j + R.D[s + 1] + q;
        const long long d = (long long)(fdr[fo[s] + x] - tfd[fo[s] + q]);
        const u32 c = (u32)(k % g);
        mn[c] = d < mn[c] ? d : mn[c];
        mx[c] = d > mx[c] ? d : mx[c];
      }
    }
    long long lo = 0, hi = 0;
    for (u32 c = 0; c < g; ++c) lo = mn[c] > lo ? mn[c] : lo, hi = mx[c] > hi ? mx[c] : hi;
    t_lo = ((u64)lo + den - 1) / den;
    t_hi = ((u64)hi + den - 1) / den;
  }
  // Brent: the tortoise jumps to the hare at powers of two; lam = blocks since the tortoise. The
  // first save waits for every stage to have started (j >= 0): from there the block map is the same
  // every block.
  __device__ __forceinline__ void init(const RRSetup &R) {
    for (int w = 0; w < MAXN; ++w) wf[w] = 0;
    for (int q = 0; q < RR_LINKS; ++q) lff[q] = lfb[q] = 0;
    for (int s = 0; s < R.S; ++s) bph[s] = bl[s] = fph[s] = fl[s] = fw[s] = fr[s] = 0;
    for (int s = 0, o = 0; s < R.S - 1; ++s) {
      fo[s] = o;
      o += R.D[s] - R.D[s + 1] + 1;
    }
    j = -(long long)R.D[0];  // the first round with an op: F_0(0)
    rounds = 0;
    do {
      block(R);
      rounds += R.Lam;
    } while (j < 0);
    save(R);
    power = 1;
    lam = 0;
  }
  // An exact repeat: every live component of each class moved by its class's first component's
  // delta since the save (stops at the first mismatch, the common case); then t_lo = t_hi = T.
  __device__ __forceinline__ bool repeated(const RRSetup &R, u64 den, u64 &t_lo, u64 &t_hi) const {
    const int S = R.S;
    const u32 g = R.g;
    long long ref[MAXN];
    bool seen[MAXN];
    for (u32 c = 0; c < g; ++c) seen[c] = false;
    auto same = [&](u32 c, long long d) {
      if (!seen[c]) {
        seen[c] = true;
        ref[c] = d;
        return true;
      }
      return d == ref[c];
    };
    for (int s = 0; s < S; ++s)
      for (int i = 0; i < R.r[s]; ++i) {
        const int w = (R.wl[s] >> (4 * i)) & 15;
        if (!same((u32)i % g, (long long)(wf[w] - tw[w]))) return false;
      }
    for (int s = 0; s < S - 1; ++s)
      for (int k = 0; k < R.lc[s]; ++k) {
        const int ql = R.lo[s] + k;
        if (!same((u32)k % g, (long long)(lff[ql] - tlf[ql])) || !same((u32)k % g, (long long)(lfb[ql] - tlb[ql])))
          return false;
      }
    for (int s = 0; s < S - 1; ++s) {
      const int len = R.D[s] - R.D[s + 1] + 1;
      for (int q = 0, x = fr[s]; q < len - 1; ++q, x = x + 1 == len ? 0 : x + 1) {
        const long long k = j + R.D[s + 1] + q;
        if (!same((u32)(k % g), (long long)(fdr[fo[s] + x] - tfd[fo[s] + q]))) return false;
      }
    }
    long long mx = 0;
    for (u32 c = 0; c < g; ++c) mx = ref[c] > mx ? ref[c] : mx;
    t_lo = t_hi = ((u64)mx + den - 1) / den;
    return true;
  }
  // One block, then the decision: the cheap exact-repeat test after every block, the growth bounds
  // (met, pruned, budget) at Brent's doublings and when the budget runs out.
  __device__ __forceinline__ int step(const RRSetup &R, u32 cap, u64 prune, u64 &t_lo, u64 &t_hi) {
    block(R);
    ++lam;
    rounds += R.Lam;
    const u64 den = (u64)lam * R.Lam;
    if (repeated(R, den, t_lo, t_hi)) return RR_MET;
    if (power == lam || rounds > cap) {
      bounds(R, den, t_lo, t_hi);
      if (t_lo == t_hi) return RR_MET;
      if (t_lo > prune) return RR_PRUNED;
      if (rounds > cap) return RR_BUDGET;
      save(R);
      power *= 2;
      lam = 0;
    }
    return RR_CONT;
  }
};

// The whole recurrence in the thread, up to `cap` rounds (S >= 2); see RRSim. *rounds_out
// (optional): rounds run.
static __device__ __noinline__ int rr_sim(const RRSetup &R, u32 cap, u64 prune, u64 &t_lo, u64 &t_hi,
                                          u32 *rounds_out) {
  RRSim sim;
  sim.init(R);
  int rc;
  do rc = sim.step(R, cap, prune, t_lo, t_hi);
  while (rc == RR_CONT);
  if (rounds_out) *rounds_out = sim.rounds;
  return rc;
}

// Node (kind, s, phase p) of the one-period event graph: F_s, B_s, forward and backward transfer of
// boundary s, for the mini-batches k = p (mod Lam); V = 4 S Lam (the transfer nodes of s = S - 1 are
// unused). Its duration, and the relaxation of its (at most two) predecessors at theta, where an
// edge's weight is -theta Lam (its token count: periods between the two mini-batches).
__device__ __forceinline__ u64 rr_dur(const RRSetup &R, int kind, int s, int ph) {
  if (kind <= 1) {
    const int w = (R.wl[s] >> (4 * (ph % R.r[s]))) & 15;
    return kind == 0 ? R.Fw[w] : R.Bw[w];
  }
  const int q = R.lo[s] + ph % R.lc[s];
  return kind == 2 ? R.tf[q] : R.tb[q];
}
template <typename Dist>
__device__ __forceinline__ long long rr_relax(const RRSetup &R, const Dist &dist, int kind, int s, int p,
                                              long long dv, long long th) {
  const int S = R.S;
  const long long Lam = R.Lam, K0 = 64ll * Lam;  // a period index far from the start
  const long long k = K0 + p;
  auto at = [&](int kk, int ss, long long ku) {
    const long long tok = k / Lam - ku / Lam;
    return dist[(kk * S + ss) * (int)Lam + (int)(ku % Lam)] + dv - th * Lam * tok;
  };
  long long best = LLONG_MIN;
  auto take = [&](long long c) { best = c > best ? c : best; };
  if (kind == 0) {
    take(at(1, s, k - (long long)R.mm[s] * R.r[s]));  // worker order: after B(k - m r)
    if (s > 0) take(at(2, s - 1, k));                   // forward transfer of boundary s - 1
  } else if (kind == 1) {
    take(at(0, s, k + (long long)(R.mm[s] - 1) * R.r[s]));  // worker order: after F(k + (m - 1) r)
    if (s < S - 1) take(at(3, s, k));                        // backward transfer of boundary s
  } else if (kind == 2) {
    take(at(0, s, k));            // after F_s(k)
    take(at(2, s, k - R.lc[s]));  // FIFO on its link
  } else {
    take(at(1, s + 1, k));  // after B_{s+1}(k)
    take(at(3, s, k - R.lc[s]));
  }
  return best;
}

// Positive cycle at theta (single thread, Gauss-Seidel passes in node order).
// A simple path weighs at most the sum of all node durations plus theta Lam negtok per edge (the
// worker-order edges B_s(k) <- F_s(k + (m - 1) r) can carry negative tokens); a larger distance
// proves a positive cycle.
__device__ __forceinline__ long long rr_path_cap(const RRSetup &R, long long th) {
  const long long V = 4ll * R.S * R.Lam;
  return (long long)R.dsum + V * (th > 0 ? th : 0) * (long long)R.Lam * R.negtok;
}
__device__ __forceinline__ bool rr_positive(const RRSetup &R, long long th, long long *dist) {
  const int S = R.S, Lam = (int)R.Lam, V = 4 * S * Lam;
  const long long cap = rr_path_cap(R, th);
  for (int v = 0; v < V; ++v) dist[v] = 0;
  for (int pass = 0; pass <= V; ++pass) {
    bool changed = false;
    for (int v = 0; v < V; ++v) {
      const int kind = v / (S * Lam), s = (v / Lam) % S, p = v % Lam;
      if (kind >= 2 && s == S - 1) continue;
      const long long c = rr_relax(R, dist, kind, s, p, (long long)rr_dur(R, kind, s, p), th);
      if (c > dist[v]) {
        dist[v] = c;
        changed = true;
        if (c > cap) return true;  // heavier than any simple path: a positive cycle
      }
    }
    if (!changed) return false;
  }
  return true;
}

// Positive cycle at theta, one warp (every lane calls it; dist: V words of the warp's shared memory).
// Lane l relaxes nodes l, l + 32, ... in place: a value read mid-pass is the old or the new one, both
// lower bounds of the pass's result, so V + 1 passes still decide (chaotic Bellman-Ford).
__device__ __forceinline__ bool rr_positive_warp(const RRSetup &R, long long th, volatile long long *dist) {
  const int S = R.S, Lam = (int)R.Lam, V = 4 * S * Lam, lane = threadIdx.x & 31;
  const long long cap = rr_path_cap(R, th);
  for (int v = lane; v < V; v += 32) dist[v] = 0;
  __syncwarp();
  for (int pass = 0; pass <= V; ++pass) {
    bool changed = false, big = false;
    for (int v = lane; v < V; v += 32) {
      const int kind = v / (S * Lam), s = (v / Lam) % S, p = v % Lam;
      if (kind >= 2 && s == S - 1) continue;
      const long long c = rr_relax(R, dist, kind, s, p, (long long)rr_dur(R, kind, s, p), th);
      if (c > dist[v]) {
        dist[v] = c;
        changed = true;
        big |= c > cap;
      }
    }
    __syncwarp();
    if (__any_sync(0xffffffffu, big)) return true;
    if (!__any_sync(0xffffffffu, changed)) return false;
  }
  return true;
}

// Predecessor `which` (0 or 1) of node v of the one-period event graph, as in rr_relax: its node id
// and the edge's token count (periods between the two mini-batches); false if v has no such edge.
__device__ __forceinline__ bool rr_pred(const RRSetup &R, int v, int which, int &u, long long &tok) {
  const int S = R.S, Lam = (int)R.Lam;
  const int kind = v / (S * Lam), s = (v / Lam) % S, p = v % Lam;
  const long long K0 = 64ll * Lam, k = K0 + p;
  int kk, ss;
  long long ku;
  if (kind == 0) {
    if (which == 0) kk = 1, ss = s, ku = k - (long long)R.mm[s] * R.r[s];
    else if (s > 0) kk = 2, ss = s - 1, ku = k;
    else return false;
  } else if (kind == 1) {
    if (which == 0) kk = 0, ss = s, ku = k + (long long)(R.mm[s] - 1) * R.r[s];
    else if (s < S - 1) kk = 3, ss = s, ku = k;
    else return false;
  } else if (kind == 2) {
    if (which == 0) kk = 0, ss = s, ku = k;
    else kk = 2, ss = s, ku = k - R.lc[s];
  } else {
    if (which == 0) kk = 1, ss = s + 1, ku = k;
    else kk = 3, ss = s, ku = k - R.lc[s];
  }
  u = (kk * S + ss) * Lam + (int)(ku % Lam);
  tok = k / Lam - ku / Lam;
  return true;
}

// An estimate of lambda_compute by Howard's policy iteration on the one-period event graph (the
// maximum cycle ratio sum(durations) / (Lam sum(tokens))), in double precision: each node keeps one
// in-edge (the policy); the policy graph's cycles give their ratios, every node the ratio of the cycle
// its policy chain reaches and a bias along the chain; a node switches to an in-edge whose source
// reaches a larger ratio, or an equal ratio with a larger bias, until none does. Only a guess for the
// exact search below (which verifies it with two Bellman-Ford tests), so rounding cannot hurt.
static __device__ __noinline__ double rr_howard(const RRSetup &R) {
  const int S = R.S, Lam = (int)R.Lam, V = 4 * S * Lam;
  unsigned char pol[RR_BF_NODES], state[RR_BF_NODES];
  double eta[RR_BF_NODES], x[RR_BF_NODES];
  int path[RR_BF_NODES];
  auto live = [&](int v) { const int kind = v / (S * Lam), s = (v / Lam) % S; return !(kind >= 2 && s == S - 1); };
  auto edge = [&](int v, int which, int &u, double &w, double &tau) {
    long long tok;
    if (!rr_pred(R, v, which, u, tok)) return false;
    const int kind = v / (S * Lam), s = (v / Lam) % S, p = v % Lam;
    w = (double)rr_dur(R, kind, s, p);
    tau = (double)Lam * (double)tok;
    return true;
  };
  for (int v = 0; v < V; ++v) pol[v] = 0;
  double best = 0.0;
  for (int it = 0; it < 64; ++it) {
    // value determination for the current policy
    for (int v = 0; v < V; ++v) state[v] = live(v) ? 0 : 2;
    for (int v0 = 0; v0 < V; ++v0) {
      if (state[v0]) continue;
      int n = 0, u = v0;
      while (state[u] == 0) {  // follow the policy backwards (to the predecessors) until a known node
        state[u] = 1;
        path[n++] = u;
        int pu;
        double w, tau;
        edge(u, pol[u], pu, w, tau);
        u = pu;
      }
      if (state[u] == 1) {  // a new cycle through u: its ratio, biases around it
        double W = 0.0, Tk = 0.0;
        int c = u;
        do {
          int pc;
          double w, tau;
          edge(c, pol[c], pc, w, tau);
          W += w;
          Tk += tau;
          c = pc;
        } while (c != u);
        const double r = Tk > 0.0 ? W / Tk : 1e300;  // a live schedule has no token-free cycle
        x[u] = 0.0;
        eta[u] = r;
        c = u;
        for (;;) {  // x(pred(c)) = x(c) - (w_c - r tau)
          int pc;
          double w, tau;
          edge(c, pol[c], pc, w, tau);
          if (pc == u) break;
          x[pc] = x[c] - (w - r * tau);
          eta[pc] = r;
          c = pc;
        }
        c = u;
        do {
          state[c] = 2;
          int pc;
          double w, tau;
          edge(c, pol[c], pc, w, tau);
          c = pc;
        } while (c != u);
      }
      for (int i = n - 1; i >= 0; --i) {  // the chain's nodes, nearest the resolved one first
        const int v = path[i];
        if (state[v] == 2) continue;
        int pv;
        double w, tau;
        edge(v, pol[v], pv, w, tau);
        eta[v] = eta[pv];
        x[v] = x[pv] + w - eta[pv] * tau;
        state[v] = 2;
      }
    }
    best = 0.0;
    for (int v = 0; v < V; ++v)
      if (live(v) && eta[v] > best) best = eta[v];
    // policy improvement
    bool changed = false;
    for (int v = 0; v < V; ++v) {
      if (!live(v)) continue;
      int u0, u1;
      double w0, t0, w1, t1;
      if (!edge(v, 1, u1, w1, t1)) continue;  // a single in-edge: nothing to choose
      edge(v, 0, u0, w0, t0);
      const double e0 = eta[u0], e1 = eta[u1];
      const double tol = 1e-12 * (e0 > e1 ? e0 : e1) + 1e-9;
      int pick = pol[v];
      if (e0 > e1 + tol) pick = 0;
      else if (e1 > e0 + tol) pick = 1;
      else {
        const double b0 = x[u0] + w0 - e0 * t0, b1 = x[u1] + w1 - e1 * t1;
        const double bt = 1e-9 * (fabs(b0) > fabs(b1) ? fabs(b0) : fabs(b1)) + 1e-6;
        if (b0 > b1 + bt) pick = 0;
        else if (b1 > b0 + bt) pick = 1;
      }
      if (pick != pol[v]) {
        pol[v] = (unsigned char)pick;
        changed = true;
      }
    }
    if (!changed) break;
  }
  return best;
}

// ceil(lambda_compute) inside the bracket t_lo <= T <= t_hi the simulation's bounds give:
// positive(t_lo - 1) holds and positive(t_hi) does not, so a binary search on theta decides it.
// (Galloping down from t_hi first was measured no faster on the C5 records: 2.2 -> 2.6 ms drain.)
template <typename Pos>
__device__ __forceinline__ u64 rr_ceil_search(u64 t_lo, u64 t_hi, Pos positive, double guess = -1.0) {
  long long lo = (long long)t_lo - 1, hi = (long long)t_hi;
  // a guess (Howard's estimate) inside the bracket is checked first: positive(g - 1) and not
  // positive(g) settle T = g with two tests; otherwise each test still halves the bracket's side
  if (guess > 0.0) {
    // lambda = p / q with q <= Lam sum(tokens) (a few thousand): a non-integral ratio sits >= 1 / q away
    // from an integer, while the double sums err by ~1e-16 relative; the nudge only absorbs that
    const long long g = (long long)ceil(guess - (1e-6 + 1e-13 * guess));
    if (g - 1 > lo && g - 1 < hi) {
      if (positive(g - 1)) lo = g - 1;
      else hi = g - 1;
    }
    if (g > lo && g < hi) {
      if (positive(g)) lo = g;
      else hi = g;
    }
  }
  while (hi - lo > 1) {
    const long long mid = lo + (hi - lo) / 2;
    if (positive(mid)) lo = mid;
    else hi = mid;
  }
  return (u64)hi;
}
__device__ __forceinline__ u64 rr_ceil_bf(const RRSetup &R, u64 t_lo, u64 t_hi) {
  long long dist[RR_BF_NODES];
  return rr_ceil_search(t_lo, t_hi, [&](long long th) { return rr_positive(R, th, dist); }, rr_howard(R));
}
__device__ __forceinline__ u64 rr_ceil_bf_warp(const RRSetup &R, u64 t_lo, u64 t_hi, volatile long long *dist) {
  // every lane computes the same estimate (no broadcast needed)
  return rr_ceil_search(t_lo, t_hi, [&](long long th) { return rr_positive_warp(R, th, dist); }, rr_howard(R));
}

// T_ns of a validated 16-byte partition under round-robin replicas, in the thread.
static __device__ __noinline__ u64 rr_time(const SmemTab &t, int S, const P8 &p, int sync) {
#if !RR_STATS
  // one worker per stage: round-robin replicas coincide with the split model (reading F-5: C-2 is
  // the case r = 1), whose closed form replaces the recurrence
  if (__popcll(p.masks) == S) return eval_closed_form<false, false, P8>(t, S, p, sync);
#endif
  RRSetup R;
  rr_setup(t, S, p, sync, R);
  if (S == 1) return umax(rr_single_stage(R), R.Tsync);
  u64 t_lo, t_hi;
  u32 rounds;
  const bool met = rr_sim(R, RR_SIM_ROUNDS, U64MAX, t_lo, t_hi, &rounds) == RR_MET;
#if RR_STATS  // diagnostics (tools/rr_stats.py): rounds simulated, bit 32 = bounds not met in the budget
  return rounds | (met ? 0ull : 1ull << 32);
#endif
  if (met || R.Tsync >= t_hi) return umax(t_lo, R.Tsync);
  return umax(rr_ceil_bf(R, t_lo, t_hi), R.Tsync);
}

}  // namespace ap
