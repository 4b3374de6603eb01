// sched.cuh — the flushed schedule variants of NEXT row f3 (reading F-3) and the
// max-plus helpers they share with the startup recurrence of row f2 (k_switch.cu).
//
// GPipe and DAPPLE's 1F1B with flush run one iteration of M
// micro-batches from an empty pipeline; T_ns = the time the last stage finishes its last backward
// (plus its gradient synchronisation if replicated). One thread evaluates one partition by running
// the schedule's own max-plus recurrence in a dependency order (no event queue):
//   GPipe   forward phase k = 0..M-1, stages ascending: F_s(k) on every replica, forward boundary s;
//           backward phase k = 0..M-1, stages descending: B_s(k), backward boundary s-1
//   DAPPLE  warm-up k = 0..n_0-1, stages ascending: F_s(k) for k < n_s = min(S - s, M);
//           rounds j = 0..M-1, stages descending: B_s(j), then F_s(j + n_s) if j + n_s < M
// In both orders every op's inputs are produced before it (B_s(j) reads backward boundary s of j,
// produced just before by stage s+1; F_s(k) reads forward boundary s-1 of k, produced earlier by
// stage s-1), each worker's ops are visited in its own list order, and each boundary's transfers in
// micro-batch order, so one "latest" value per boundary, one free time per worker and one free time per
// boundary direction (its links are used by no other boundary) reproduce the ready-driven execution
// exactly.
#pragma once
#include "eval.cuh"
#include "chimera.cuh"
#include "rr.cuh"

namespace ap {

// T_ns of one flushed iteration (GPipe or DAPPLE) of a validated partition (P8 or the wide P16). Loops
// run over the actual stages and over each stage's own workers (its mask bits), with the per-worker
// and per-stage state in small arrays: the unrolled form with every worker slot predicated in every
// stage step (S x N slot visits per round, registers for 16-byte records, spills for wide ones) was
// slower at both widths (B200, 1M records, M = 8: GPipe 0.70 -> 0.56 ms, DAPPLE 0.68 -> 0.64; wide
// GPipe + recompute 6.0 -> 2.2, wide DAPPLE 9.0 -> 2.4; BERT-24 searches GPipe 1.8 -> 1.2, DAPPLE
// 3.5 -> 2.2).
template <int SCHED, typename P>
__device__ __forceinline__ u64 flush_makespan(const SmemTab &t, int S, const P &p, const ModelP &m) {
  static_assert(SCHED == SCHED_GPIPE || SCHED == SCHED_DAPPLE, "flushed schedules only");
  constexpr int MS = P::MS, MN = P::MN;
  const int M = (int)m.M;
  u64 Fd[MN], Bd[MN], wf[MN];
  u32 msk[MS];
  u64 dF[MS], dB[MS], lfF[MS], lfB[MS], fdl[MS], last[MS];
  for (int s = 0; s < S; ++s) {
    const u32 mask = p.mask(s);
    msk[s] = mask;
    const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
    const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
    const DivR<MN> dv((u32)__popc(mask), t.dv);
    for (u32 mm = mask; mm; mm &= mm - 1) {
      const int w = __ffs(mm) - 1;
      Fd[w] = dv.ceil(t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a]);
      Bd[w] = dv.ceil(t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a]);
      if (SCHED == SCHED_GPIPE && m.recompute) Bd[w] += Fd[w];  // the backward op re-runs the forward
      wf[w] = 0;
    }
    // One boundary's transfers all start at its barrier and use links no other boundary uses, so its
    // completion over the micro-batches is that of a single FIFO server with the longest transfer:
    // max_p lf_p(k) with lf_p(k) = max(bar_k, lf_p(k-1)) + d_p equals max_j (bar_j + (k-j+1) max_p d_p)
    // (bar_k is non-decreasing in k). Per boundary and direction: its longest transfer and free time.
    dF[s] = dB[s] = lfF[s] = lfB[s] = fdl[s] = last[s] = 0;
    if (s < S - 1) boundary_cf_cb<MN>(t, p.cut(s), mask, p.mask(s + 1), dF[s], dB[s]);
  }
  // F_s(k) on every replica of stage s, then forward boundary s (as flush_makespan)
  auto fwd = [&](int s) {
    const u64 ready = s == 0 ? 0ull : fdl[s - 1];
    u64 bar = 0;
    for (u32 mm = msk[s]; mm; mm &= mm - 1) {
      const int w = __ffs(mm) - 1;
      wf[w] = umax(wf[w], ready) + Fd[w];
      bar = umax(bar, wf[w]);
    }
    if (s < S - 1) {
      lfF[s] = umax(bar, lfF[s]) + dF[s];
      fdl[s] = lfF[s];
    }
  };
  // B_s(k) on every replica of stage s (input: bd), then backward boundary s-1 (into bd)
  auto bwd = [&](int s, int k, u64 &bd) {
    const u64 ready = s == S - 1 ? 0ull : bd;
    u64 bar = 0;
    for (u32 mm = msk[s]; mm; mm &= mm - 1) {
      const int w = __ffs(mm) - 1;
      wf[w] = umax(wf[w], ready) + Bd[w];
      bar = umax(bar, wf[w]);
    }
    if (s > 0) {
      lfB[s - 1] = umax(bar, lfB[s - 1]) + dB[s - 1];
      bd = lfB[s - 1];
    }
    if (k == M - 1) last[s] = bar;
  };
  if (SCHED == SCHED_GPIPE) {
    for (int k = 0; k < M; ++k)
      for (int s = 0; s < S; ++s) fwd(s);
    for (int k = 0; k < M; ++k) {
      u64 bd = 0;
      for (int s = S - 1; s >= 0; --s) bwd(s, k, bd);
    }
  } else {
    const int nw = S < M ? S : M;  // n_0 = min(S, M) warm-up rounds
    for (int k = 0; k < nw; ++k)
      for (int s = 0; s < S; ++s)
        if (k < S - s) fwd(s);  // k < n_s = min(S - s, M) (k < M already)
    for (int j = 0; j < M; ++j) {
      u64 bd = 0;
      for (int s = S - 1; s >= 0; --s) {
        bwd(s, j, bd);
        if (j + (S - s) < M) fwd(s);  // F_s(j + n_s), n_s = S - s when j + n_s < M
      }
    }
  }
  u64 T = 0;
  for (int s = 0; s < S; ++s) {
    u64 x = last[s];
    if (__popc(msk[s]) >= 2) {
      const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
      const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
      x += sync_time<MN>((int)m.sync, t.PP[e + 1] - t.PP[a], msk[s], t.tau, t.dv);
    }
    T = umax(T, x);
  }
  return T;
}

// A lower bound on T_ns under a flushed schedule (GPipe, DAPPLE) or Chimera, for the pruned searches:
// GPipe / DAPPLE: worker w of stage s runs its M forwards and M backwards one after another, after
// micro-batch 0 has crossed stages 0..s-1 (each stage's slowest replica, then the boundary) and before
// micro-batch M-1's gradient crosses back to stage 0:
//   T >= sum_{u<s} (maxF_u + dF_u) + M (F_w + B_w) + sum_{u<s} (dB_u + maxB_u);
// plus each schedule's fill term (DAPPLE: micro-batch 0's round trip beyond s before B_s(0); GPipe:
// the last stage's M forwards before any backward), below;
// Chimera: worker g runs ceil(M/2) micro-batches of its down stage and floor(M/2) of its up stage.
// UINT64_MAX for a record the model refuses (Chimera: a replicated stage).
template <int MODE, typename P>
__device__ __forceinline__ u64 model_lower(const SmemTab &t, int S, const P &p, const ModelP &m) {
  constexpr int MN = P::MN;
  const u64 M = m.M;
  if constexpr (MODE == SCHED_CHIMERA) {
    const u64 Md = (M + 1) / 2, Mu = M / 2;
    u64 lb = 0;
    for (int g = 0; g < S; ++g) {
      const u32 mask = p.mask(g);
      if (__popc(mask) != 1) return U64MAX;
      const int w = __ffs(mask) - 1, su = S - 1 - g;
      const int a = (g == 0) ? 0 : p.cut(g - 1) + 1, e = (g == S - 1) ? t.L - 1 : p.cut(g);
      const int au = (su == 0) ? 0 : p.cut(su - 1) + 1, eu = (su == S - 1) ? t.L - 1 : p.cut(su);
      const u64 *F = t.PF + w * t.Lp1, *B = t.PB + w * t.Lp1;
      lb = umax(lb, Md * (F[e + 1] - F[a] + B[e + 1] - B[a]) + Mu * (F[eu + 1] - F[au] + B[eu + 1] - B[au]));
    }
    return lb;
  } else {
    static_assert(MODE == SCHED_GPIPE || MODE == SCHED_DAPPLE, "flushed schedules and Chimera");
    // per stage u: maxF_u, maxB_u (the slowest replica: a stage op ends at its replicas' barrier),
    // cf_u, cb_u (boundary u). tot = one micro-batch's whole round trip; pre = the crossing to stage s
    // and back; fwd = the forward crossing to stage S - 1.
    u64 lb = 0, pre = 0, tot = 0, fwd = 0, sumB = 0, sumCB = 0, dap = 0, gmaxB = 0, qlast = 0;
    for (int s = 0; s < S; ++s) {
      const u32 mask = p.mask(s);
      const int a = (s == 0) ? 0 : p.cut(s - 1) + 1, e = (s == S - 1) ? t.L - 1 : p.cut(s);
      const DivR<MN> dv((u32)__popc(mask), t.dv);
      const u64 ns = (u64)(S - s) < M ? (u64)(S - s) : M;  // DAPPLE's warm-up forwards
      u64 mF = 0, mB = 0, work = 0, kd = 0, q = 0;
      for (u32 mm = mask; mm; mm &= mm - 1) {
        const int w = __ffs(mm) - 1;
        const u64 Fw = dv.ceil(t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a]);
        u64 Bw = dv.ceil(t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a]);
        if (MODE == SCHED_GPIPE && m.recompute) Bw += Fw;
        mF = umax(mF, Fw);
        mB = umax(mB, Bw);
        work = umax(work, Fw + Bw);
        kd = umax(kd, M * Bw + (M - ns) * Fw);
        q = umax(q, M * Fw + Bw);
      }
      // a worker's M forwards and backwards between the crossings (both schedules)
      lb = umax(lb, pre + M * work);
      tot += mF + mB;
      dap = umax(dap, kd - mB);  // kd >= M mB >= mB
      if (s < S - 1) {
        u64 cf, cb;
        boundary_cf_cb<MN>(t, p.cut(s), mask, p.mask(s + 1), cf, cb);
        pre += mF + cf + cb + mB;
        tot += cf + cb;
        fwd += mF + cf;
        sumB += mB;
        sumCB += cb;
        gmaxB = umax(gmaxB, mB);
      } else {
        qlast = q;
      }
    }
    if (MODE == SCHED_DAPPLE) {
      // a worker of stage s starts B_s(0) after micro-batch 0's round trip beyond s and then still
      // runs M backwards and M - n_s forwards; micro-batch M - 1's gradient crosses back:
      //   T >= tot - maxB_s + M B_w + (M - n_s) F_w
      lb = umax(lb, tot + dap);
    } else if (S > 1) {
      // GPipe: B_s(0) (s < S - 1) waits for the last stage's M forwards and the backward chain down
      // to s; then the worker runs M backwards and the gradient crosses back to stage 0:
      //   T >= fwd + max_w(M F_w + B_w)[S - 1] + sum_{u < S-1} cb_u + sum_{u < S-1, u != s} maxB_u + M maxB_s
      lb = umax(lb, fwd + qlast + sumCB + sumB + (M - 1) * gmaxB);
    }
    return lb;
  }
}

// T_ns of a validated partition under the model (rows f3, f4): MODE = the schedule, fixed per kernel.
// Round-robin replicas (SCHED_RR) are defined for 16-byte records (the host refuses wide ones).
template <int MODE, bool P32, typename P>
__device__ __forceinline__ u64 model_time(const SmemTab &t, int S, const P &p, const ModelP &m) {
  if constexpr (MODE == SCHED_RR) {
    if constexpr (P::MS == 8) return rr_time(t, S, p, (int)m.sync);
    else return U64MAX;
  }
  if constexpr (MODE == SCHED_CHIMERA) return chimera_time<P>(t, S, p, m);  // row f3, reading F-6
  if (MODE == SCHED_PIPEDREAM) return eval_closed_form<P32, false, P>(t, S, p, (int)m.sync);
  if (MODE == SCHED_2BW) return eval_closed_form<false, true, P>(t, S, p, (int)m.sync, m.M);
  constexpr int FS = (MODE == SCHED_PIPEDREAM || MODE == SCHED_2BW || MODE == SCHED_RR || MODE == SCHED_CHIMERA)
                         ? SCHED_GPIPE : MODE;
  return flush_makespan<FS, P>(t, S, p, m);
}

}  // namespace ap
