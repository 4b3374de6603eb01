// k_search.cu — exhaustive search (autopipe_search_optimum), rows a3-a8 for the general space:
// combinatorial unranking of the global index (SPEC.md §5), lexicographic successor, the closed form
// per candidate, and a warp -> block -> grid lexicographic (time, index) argmin.
//
// The paper enumerates candidate partitions and scores each with its speed model
// (PAPER.md:896-899); here every candidate of [begin, end) is scored exactly. Launch: a persistent
// grid (a multiple of the SM count) of 256-thread blocks; thread t owns the contiguous index range
// [begin + t*k, begin + (t+1)*k): it unranks its first index once, then steps with the lexicographic
// successor (the last cut moves fastest). Each block writes its (T, index, count); k_finalize reduces
// the blocks and decodes the winner. The argmin is the lexicographic minimum of (T, index), so the
// result does not depend on the grid, the block count or the number of GPUs.
#include "binom.cuh"
#include "eval.cuh"
#include "internal.h"
#include "sched.cuh"
#include "rr.cuh"

namespace ap {

// Space-generic pieces: a 16-byte space (S, N <= 8: P8, subsets packed in one u64, binomial rows of 9
// columns in shared memory) or a wide one (row f4; S, N <= 16: P16, Pk2 subsets, 17 columns).
template <typename P>
struct SpaceT;
template <>
struct SpaceT<P8> {
  typedef u64 PK;
  static constexpr int BK = BK8;
  __device__ static bool next(PK &p, int k, int n) { return lex_next_packed(p, k, n); }
  __device__ static P8 part(u64 cuts, u64 masks) { return P8{cuts, masks}; }
};
template <>
struct SpaceT<P16> {
  typedef Pk2 PK;
  static constexpr int BK = BINOM_K;
  __device__ static bool next(PK &p, int k, int n) { return lex_next_pk2(p, k, n); }
};

template <typename PK>
__device__ __forceinline__ PK first_subset(int k) {
  PK p;
  pk_zero(p);
  for (int j = 0; j < k; ++j) pk_or(p, j, j);
  return p;
}

__device__ __forceinline__ int comp_k(const SearchSpace &sp, int S) { return (sp.flags & 1) ? S - 1 : S; }
__device__ __forceinline__ int comp_n(const SearchSpace &sp) { return (sp.flags & 1) ? sp.N - 1 : sp.N; }

// The partition of (S, composition Rp, cut set): contiguous placement, stage s gets workers
// [R_{s-1}, R_s) (reading C-11).
template <typename P, typename PK>
__device__ __forceinline__ P part_from(const SearchSpace &sp, int S, const PK &Rp, const PK &cuts) {
  const bool all = sp.flags & 1;
  P p;
  int prev = 0;
  if constexpr (P::MS == 8) {
    p.cuts = cuts;
    p.masks = 0;
  } else {
    p.c[0] = cuts.lo;
    p.c[1] = cuts.hi;
    p.m[0] = p.m[1] = p.m[2] = p.m[3] = 0;
  }
#pragma unroll
  for (int s = 0; s < P::MS; ++s) {
    if (s < S) {
      const int R = (all && s == S - 1) ? sp.N : pk_get(Rp, s) + 1;
      const u32 m = ((1u << R) - 1u) & ~((1u << prev) - 1u);
      if constexpr (P::MS == 8) p.masks |= (u64)m << (8 * s);
      else p.m[s >> 2] |= (u64)m << (16 * (s & 3));
      prev = R;
    }
  }
  return p;
}

// global index -> (S, composition, cut set), against a binomial table in shared memory
// (fixed-length binary searches, no divergence)
template <int BK, typename PK>
__device__ __forceinline__ void unrank_global_smem(const SearchSpace &sp, u64 idx, int &S, PK &Rp, PK &cuts,
                                                   const u64 *Bn) {
  S = sp.s_min;
  while (S < sp.s_max && idx >= sp.off[S + 1]) ++S;
  const u64 rem = idx - sp.off[S];
  const u64 rho = rem / sp.ncut[S], kappa = rem % sp.ncut[S];
  Rp = lex_unrank_smem<BK, PK>(rho, comp_k(sp, S), comp_n(sp), Bn);
  cuts = lex_unrank_smem<BK, PK>(kappa, S - 1, sp.L - 1, Bn);
}

#ifndef GEN_MINB
#define GEN_MINB 3  // B200: 3 blocks per SM (C2 VGG-16 0.22 -> 0.18 ms) beat 1 and 2
#endif
// NARROW (PipeDream, dense launches of a host-classified state): the 32-bit closed form of k_eval
template <int NT, bool P32, int MODE, typename P, bool NARROW = false>
__global__ void __launch_bounds__(NT, GEN_MINB) k_search_generic(DevTables g, SearchSpace sp, u64 begin, u64 end,
                                                                 u64 per_thread, BlockOut *out, ModelP m, int gate,
                                                                 u64 *gbest = nullptr) {
  if (gate >= 0 && state_gated_out(g, gate, out)) return;  // see state_gated_out
  typedef SpaceT<P> SP;
  typedef typename SP::PK PK;
  constexpr int BK = SP::BK;
  // flushed schedules and Chimera: candidates decided by a lower bound against the best so far
  constexpr bool PRUNED = MODE == SCHED_GPIPE || MODE == SCHED_DAPPLE || MODE == SCHED_CHIMERA;
  extern __shared__ u64 sm[];
  // binomial rows n <= L (n = N <= 16 <= L + 1 for the compositions too) after the state tables
  u64 *Bn = sm + smem_words(g.L, g.N, NARROW);
  const int nb = ((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK;
  for (int i = threadIdx.x; i < nb; i += NT) Bn[i] = g_binom[i / BK][i % BK];
  const SmemTab t = stage_tables<NARROW>(g, sm);  // ends with __syncthreads()
  const u64 gtid = (u64)blockIdx.x * NT + threadIdx.x;
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0;
  const u64 span = end - begin;
  if (gtid < (span + per_thread - 1) / per_thread) {
    const u64 i0 = begin + gtid * per_thread;
    const u64 i1 = (end - i0 < per_thread) ? end : i0 + per_thread;
    int S;
    PK Rp, cuts;
    unrank_global_smem<BK>(sp, i0, S, Rp, cuts, Bn);
    P p = part_from<P>(sp, S, Rp, cuts);
    for (u64 i = i0; i < i1; ++i) {
      u64 T;
      if constexpr (NARROW) {
        T = eval_closed_form_n<P32, P>(t, S, p, (int)m.sync);
      } else if constexpr (PRUNED) {
        // a candidate whose lower bound exceeds theta cannot be the lexicographic minimum: theta =
        // the thread's best - 1 (its later indices lose ties) or the launch's best (the T of a real
        // candidate: a strictly greater bound loses whatever the index)
        const u64 theta = umin(bestT - 1, *(volatile u64 *)gbest);
        T = model_lower<MODE, P>(t, S, p, m) > theta ? U64MAX : model_time<MODE, P32>(t, S, p, m);
      } else {
        T = model_time<MODE, P32>(t, S, p, m);
      }
      if (T < bestT) {  // indices increase along the thread's range: strict < keeps the first
        bestT = T;
        bestI = i;
        if constexpr (PRUNED) atomicMin((unsigned long long *)gbest, T);
      }
      ++cnt;
      if (i + 1 == i1) break;
      if (!SP::next(cuts, S - 1, sp.L - 1)) {  // cut set exhausted: next composition
        cuts = first_subset<PK>(S - 1);
        if (!SP::next(Rp, comp_k(sp, S), comp_n(sp))) {  // compositions exhausted: next S
          ++S;
          if (S > sp.s_max) break;
          Rp = first_subset<PK>(comp_k(sp, S));
          cuts = first_subset<PK>(S - 1);
        }
      }
      p = part_from<P>(sp, S, Rp, cuts);
    }
  }
  block_minloc_store<NT>(bestT, bestI, cnt, out + blockIdx.x);
}

// ---------------------------------------------------------------------------------------------
// PipeDream search by prefix thresholds (rows a3-a8 for every composition; SPEC.md §4-§5).
//
// A thread walks its contiguous index range in lexicographic order, which is a depth-first walk over
// the cuts (the last cut moves fastest). It decides, per candidate, whether T <= theta, theta = its
// best T so far minus 1 (strict: its indices increase) or the block's best T (non-strict: ties keep
// the lower index), whichever is lower; only a candidate that passes gets its exact T (the full
// closed form), so every candidate is decided exactly and the thread's result is its lexicographic
// (T, index) minimum.
// The decision needs no division by segment lengths: T <= theta iff every single term is <= theta
// and every segment W(s,t) <= theta (t - s + 1). Scanning stages left to right, the segments still
// open after stage t are summarised by one number (the parametric DP of SPEC.md §A.6):
//   O_t = max over s <= t of (X_s + sum_{s<v<=t} Y_v + sum_{s<=v<t} Z_v - theta (t - s + 1))
//       = max(X_t - theta, O_{t-1} + Z_{t-1} + Y_t - theta),
// and the segments closing at t fit iff O_{t-1} + Z_{t-1} + X_t - theta <= 0. O_t of the prefix
// stages 0..S-3 is kept per level, so a lexicographic step recomputes only the levels whose cut
// moved; along a row (the last cut e) only stage S-2 = [a, e], boundary S-2 and stage S-1 change.
// A prefix that fails decides every candidate below it at once (they all contain the failing
// term): the walk jumps over that subtree, whose size is 1 + sum_{j > t} C(L - 2 - e_j, S - 1 - j)
// from the current position. Along a row, stage S-2 only grows with e (its X, Y, sync terms are
// non-decreasing), so a failure there decides the rest of the row.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ void pk_set(u64 &v, int i, int x) {
  v = (v & ~(0xFFull << (8 * i))) | ((u64)x << (8 * i));
}
__device__ __forceinline__ void pk_set(Pk2 &v, int i, int x) {
  if (i < 8) pk_set(v.lo, i, x);
  else pk_set(v.hi, i - 8, x);
}

// lexicographic successor of the k-subset `c` of {0..n-1} moving only positions <= lv; false if none
template <typename PK>
__device__ __forceinline__ bool cut_next_from(PK &c, int lv, int k, int n, int &changed) {
  for (int i = lv; i >= 0; --i) {
    const int x = pk_get(c, i);
    if (x < n - k + i) {
      for (int j = i; j < k; ++j) pk_set(c, j, x + 1 + (j - i));
      changed = i;
      return true;
    }
  }
  return false;
}

__device__ __forceinline__ u32 range_mask(int lo, int hi) {  // workers [lo, hi)
  return ((hi >= 32 ? 0xFFFFFFFFu : ((1u << hi) - 1u))) & ~((1u << lo) - 1u);
}

template <typename PK>
__device__ __forceinline__ u32 stage_mask(const SearchSpace &sp, int S, const PK &Rp, int s) {
  const bool all = sp.flags & 1;
  const int R = (all && s == S - 1) ? sp.N : pk_get(Rp, s) + 1;
  const int R0 = (s == 0) ? 0 : pk_get(Rp, s - 1) + 1;
  return range_mask(R0, R);
}

// stage [a, e] on the replicas `mask`: X = max(F' + B'), Y = max F' + max B', AR = its sync term
template <int MN>
__device__ __forceinline__ void stage_cost(const SmemTab &t, int a, int e, u32 mask, int sync, u64 &X, u64 &Y,
                                           u64 &AR) {
  const u32 r = __popc(mask);
  if (r == 1) {  // one worker: no division, no sync
    const int w = __ffs(mask) - 1;
    X = t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a];
    Y = t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a];
    X += Y;
    Y = X;
    AR = 0;
    return;
  }
  const DivR<MN> dv(r, t.dv);
  u32 m = mask;
  u64 fm = 0, bm = 0, xm = 0;
  while (m) {
    const int w = __ffs(m) - 1;
    m &= m - 1;
    const u64 F = dv.ceil(t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a]);
    const u64 B = dv.ceil(t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a]);
    fm = umax(fm, F);
    bm = umax(bm, B);
    xm = umax(xm, F + B);
  }
  X = xm;
  Y = fm + bm;
  AR = (r >= 2) ? sync_time<MN>(sync, t.PP[e + 1] - t.PP[a], mask, t.tau, t.dv) : 0ull;
}

#ifndef DFS_MINB
#define DFS_MINB 2  // resident blocks per SM of the threshold walk
#endif
#ifndef DFS_MINCH
#define DFS_MINCH 16  // candidates per chunk at least
#endif

// Dynamic schedule of the walk: chunks of the shard drawn from a global counter (so a thread whose
// chunk collapses into a few subtree jumps takes the next one), and the grid's best exact T so far
// (a bound every thread decides against, non-strictly). Reset by the launcher before each launch.
struct DfsSched {
  unsigned int next, pad;
  unsigned long long best;
};

template <int NT, typename P>
__global__ void __launch_bounds__(NT, DFS_MINB) k_search_dfs(DevTables g, SearchSpace sp, u64 begin, u64 end,
                                                             u64 chunk, BlockOut *out, ModelP m, DfsSched *ds,
                                                             int gate) {
  if (gate >= 0 && state_gated_out(g, gate, out)) return;  // see state_gated_out
  typedef SpaceT<P> SP;
  typedef typename SP::PK PK;
  constexpr int BK = SP::BK, MN = P::MN, MS = P::MS;
  extern __shared__ u64 sm[];
  __shared__ unsigned long long s_best;  // the block's best exact T so far
  u64 *Bn = sm + smem_words(g.L, g.N);
  const int nb = ((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK;
  for (int i = threadIdx.x; i < nb; i += NT) Bn[i] = g_binom[i / BK][i % BK];
  if (threadIdx.x == 0) s_best = U64MAX;
  const SmemTab t = stage_tables(g, sm);  // ends with __syncthreads()
  const int L = t.L, n = L - 1, sync = (int)m.sync;
  const u64 nchunks = (end - begin + chunk - 1) / chunk;
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0;
  long long O[MS];
  for (;;) {
    const u64 c = atomicAdd(&ds->next, 1u);
    if (c >= nchunks) break;
    const u64 i0 = begin + c * chunk;
    const u64 i1 = (end - i0 < chunk) ? end : i0 + chunk;
    cnt += i1 - i0;
    u64 gbest = *(volatile unsigned long long *)&ds->best;  // refreshed per chunk
    int S;
    PK Rp, cuts;
    unrank_global_smem<BK>(sp, i0, S, Rp, cuts, Bn);
    long long th = 0;
    bool have_th = false;
    int valid = 0;  // levels [0, valid) of O are computed for the current cuts and th
    u64 idx = i0;
    auto exact = [&]() -> u64 {
      const P p = part_from<P>(sp, S, Rp, cuts);
      return eval_closed_form<false, false, P>(t, S, p, sync);
    };
    auto next_comp = [&]() -> bool {  // the next composition (or S), first cut set
      cuts = first_subset<PK>(S - 1);
      valid = 0;
      if (SP::next(Rp, comp_k(sp, S), comp_n(sp))) return true;
      ++S;
      if (S > sp.s_max) return false;
      Rp = first_subset<PK>(comp_k(sp, S));
      cuts = first_subset<PK>(S - 1);
      return true;
    };
    auto after_level = [&](int lv) -> bool {  // past the subtree of level lv (-1: of the composition)
      int ch = 0;
      if (lv >= 0 && cut_next_from(cuts, lv, S - 1, n, ch)) {
        if (ch < valid) valid = ch;
        return true;
      }
      return next_comp();
    };
    auto improve = [&](u64 T) {
      if (T < bestT) {
        bestT = T;
        bestI = idx;
        atomicMin(&s_best, (unsigned long long)T);
        if (T < gbest) {
          atomicMin(&ds->best, (unsigned long long)T);
          gbest = T;
        }
      }
    };
    bool more = true;
    while (more) {
      // threshold: own best - 1 (strict: own indices increase), or a shared best (non-strict: ties
      // keep the lower index) when lower
      {
        const u64 sb = umin(*(volatile unsigned long long *)&s_best, gbest);
        if (bestT == U64MAX && sb == U64MAX) {  // no bound yet: this candidate is scored exactly
          improve(exact());
          ++idx;
          more = idx < i1 && after_level(S - 2);
          continue;
        }
        long long nth = (bestT == U64MAX) ? (long long)(1ull << 62) : (long long)bestT - 1;
        if (sb < (u64)nth) nth = (long long)sb;
        if (!have_th || nth != th) {
          th = nth;
          have_th = true;
          valid = 0;
        }
      }
      // prefix levels valid .. S-3
      int dead = -1;
      for (int lv = valid; lv <= S - 3; ++lv) {
        const int a = (lv == 0) ? 0 : pk_get(cuts, lv - 1) + 1;
        const int e = pk_get(cuts, lv);
        const u32 mk = stage_mask(sp, S, Rp, lv);
        u64 X, Y, AR;
        stage_cost<MN>(t, a, e, mk, sync, X, Y, AR);
        bool ok = (long long)X <= th && (long long)AR <= th;
        long long o = (long long)X - th;
        if (lv > 0) {
          const u32 mp = stage_mask(sp, S, Rp, lv - 1);
          u64 cf, cb;
          boundary_cf_cb<MN>(t, a - 1, mp, mk, cf, cb);
          const long long Z = (long long)(cf + cb);
          ok &= (long long)umax(cf, cb) <= th && O[lv - 1] + Z + (long long)X - th <= 0;
          const long long o2 = O[lv - 1] + Z + (long long)Y - th;
          o = o > o2 ? o : o2;
        }
        if (!ok) {
          dead = lv;
          break;
        }
        O[lv] = o;
        valid = lv + 1;
      }
      if (dead >= 0) {
        // every candidate below the failing prefix is decided: jump over the rest of its subtree
        u64 rem = 1;
        for (int j = dead + 1; j <= S - 2; ++j) rem += Bn[(L - 2 - pk_get(cuts, j)) * BK + (S - 1 - j)];
        if (rem >= i1 - idx) break;
        idx += rem;
        more = after_level(dead);
        continue;
      }
      if (S == 1) {  // one stage: one candidate per composition
        u64 X, Y, AR;
        stage_cost<MN>(t, 0, L - 1, stage_mask(sp, 1, Rp, 0), sync, X, Y, AR);
        if ((long long)X <= th && (long long)AR <= th) improve(exact());
        ++idx;
        more = idx < i1 && after_level(-1);
        continue;
      }
      // the row: the last cut e sweeps; Pz = the excess of the segments open after stage S-3 plus
      // boundary S-3 into stage S-2
      const u32 m2 = stage_mask(sp, S, Rp, S - 2), ml = stage_mask(sp, S, Rp, S - 1);
      const int a2 = (S >= 3) ? pk_get(cuts, S - 3) + 1 : 0;
      long long Pz = -(1ll << 62);
      if (S >= 3) {
        const u32 mp = stage_mask(sp, S, Rp, S - 3);
        u64 cf, cb;
        boundary_cf_cb<MN>(t, a2 - 1, mp, m2, cf, cb);
        if ((long long)umax(cf, cb) > th) {  // the whole row fails on boundary S-3
          const u64 rem = (u64)(L - 1 - pk_get(cuts, S - 2));
          if (rem >= i1 - idx) break;
          idx += rem;
          more = after_level(S - 3);
          continue;
        }
        Pz = O[S - 3] + (long long)(cf + cb);
      }
      int e = pk_get(cuts, S - 2);
      bool moved = false;  // a candidate passed: theta drops, the prefix is re-derived
      for (; e <= L - 2; ++e, ++idx) {
        if (idx >= i1) break;
        u64 X2, Y2, AR2;
        stage_cost<MN>(t, a2, e, m2, sync, X2, Y2, AR2);
        if ((long long)X2 > th || (long long)AR2 > th || Pz + (long long)X2 - th > 0) {
          // stage S-2 only grows with e: the rest of the row fails
          idx += (u64)(L - 1 - e);
          e = L - 1;
          break;
        }
        u64 cf, cb;
        boundary_cf_cb<MN>(t, e, m2, ml, cf, cb);
        if ((long long)umax(cf, cb) > th) continue;
        u64 Xl, Yl, ARl;
        stage_cost<MN>(t, e + 1, L - 1, ml, sync, Xl, Yl, ARl);
        const long long o2a = (long long)X2 - th, o2b = Pz + (long long)Y2 - th;
        const long long O2 = o2a > o2b ? o2a : o2b;
        if ((long long)Xl > th || (long long)ARl > th || O2 + (long long)(cf + cb) + (long long)Xl - th > 0) continue;
        // passed: T <= th < bestT, the thread's new best
        pk_set(cuts, S - 2, e);
        improve(exact());
        ++idx;
        ++e;
        moved = true;
        break;
      }
      if (idx >= i1) break;
      if (moved && e <= L - 2) {  // continue the row from e under the new threshold
        pk_set(cuts, S - 2, e);
        continue;
      }
      more = after_level(S - 3);  // row done: the next prefix
    }
  }
  block_minloc_store<NT>(bestT, bestI, cnt, out + blockIdx.x);
}

template <int NT, typename P>
static void run_search_generic(unsigned nbk, size_t smem, cudaStream_t st, const DevTables &g, const SearchSpace &sp,
                               u64 begin, u64 end, u64 pt, BlockOut *out, const ModelP &m, int path32, void *sched) {
  // the pruned schedules keep the launch's best T in the first word of their schedule slot
  u64 *gbest = (u64 *)sched;
  if (m.sched == SCHED_GPIPE || m.sched == SCHED_DAPPLE || m.sched == SCHED_CHIMERA)
    cudaMemsetAsync(gbest, 0xFF, sizeof(u64), st);
  switch (m.sched) {
    case SCHED_2BW: k_search_generic<NT, false, SCHED_2BW, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1); break;
    case SCHED_GPIPE: k_search_generic<NT, false, SCHED_GPIPE, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1, gbest); break;
    case SCHED_DAPPLE: k_search_generic<NT, false, SCHED_DAPPLE, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1, gbest); break;
    case SCHED_RR: k_search_generic<NT, false, SCHED_RR, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1); break;
    case SCHED_CHIMERA: k_search_generic<NT, false, SCHED_CHIMERA, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1, gbest); break;
    default: {  // PipeDream: the threshold walk (64-bit; the state's integer path does not matter)
      DfsSched *ds = (DfsSched *)sched;
      if (path32 >= 0) {
        cudaMemsetAsync(ds, 0, sizeof(DfsSched), st);
        cudaMemsetAsync(&ds->best, 0xFF, sizeof(u64), st);
        k_search_dfs<NT, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, ds, -1);
      } else {  // path chosen on the device (state_gated_out): both, writing disjoint block ranges
        cudaMemsetAsync(ds, 0, 2 * sizeof(DfsSched), st);
        cudaMemsetAsync(&ds[0].best, 0xFF, sizeof(u64), st);
        cudaMemsetAsync(&ds[1].best, 0xFF, sizeof(u64), st);
        k_search_dfs<NT, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, ds, 1);
        k_search_dfs<NT, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out + nbk, m, ds + 1, 0);
      }
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Round-robin replicas search (row f4, 16-byte spaces). Every candidate is decided exactly, but most
// are decided by bounds: a candidate whose lower bound exceeds theta cannot be the lexicographic
// minimum (theta = min(the thread's best - 1, the launch's best so far); the launch's best is the T
// of a real candidate, so a strictly greater bound is safe whatever the indices). The lower bound is
// first the single-resource one (rr_lower, Tsync), then the recurrence's own growth bound, which
// stops the simulation as soon as it passes theta. A candidate the recurrence has not pinned within
// RR_DEFER_ROUNDS rounds goes to the deferral queue with its bracket; the drain kernel finishes the
// queued candidates that can still win (bracket low <= the launch's best) with warp-parallel
// Bellman-Ford and contributes one (T, index) per block to the final reduction.
// Launch: one wave of 256-thread blocks drawing chunks of consecutive indices from a counter (the
// costs of neighbouring candidates vary together); a thread unranks its chunk's first index once,
// then steps with the lexicographic successor.
struct RRSearchSched {
  u64 best;   // the launch's best T so far (atomicMin)
  u32 chunk;  // next chunk
  u32 pad;
};
constexpr int RR_NT = 256;
__global__ void __launch_bounds__(RR_NT, 2) k_search_rr(DevTables g, SearchSpace sp, u64 begin, u64 end, u64 chunk,
                                                        BlockOut *out, ModelP m, RRSearchSched *rs, RRQueue q) {
  typedef SpaceT<P8> SP;
  typedef typename SP::PK PK;
  constexpr int BK = SP::BK;
  extern __shared__ u64 sm[];
  u64 *Bn = sm + smem_words(g.L, g.N);
  const int nb = ((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK;
  for (int i = threadIdx.x; i < nb; i += RR_NT) Bn[i] = g_binom[i / BK][i % BK];
  const SmemTab t = stage_tables<false>(g, sm);  // ends with __syncthreads()
  const int sync = (int)m.sync;
  const u64 span = end - begin, nch = (span + chunk - 1) / chunk;
  volatile u64 *gbest = &rs->best;
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0;
  for (;;) {
    const u64 c = atomicAdd(&rs->chunk, 1u);
    if (c >= nch) break;
    const u64 i0 = begin + c * chunk, i1 = (end - i0 < chunk) ? end : i0 + chunk;
    int S;
    PK Rp, cuts;
    unrank_global_smem<BK>(sp, i0, S, Rp, cuts, Bn);
    for (u64 i = i0; i < i1; ++i) {
      const P8 p = part_from<P8>(sp, S, Rp, cuts);
      const u64 gb = *gbest;
      const u64 theta = umin(bestT - 1, gb);  // bestT = U64MAX: no own best yet
      u64 T = U64MAX;
      if (__popcll(p.masks) == S) {  // one worker per stage: the split model's closed form (F-5)
        T = eval_closed_form<false, false, P8>(t, S, p, sync);
      } else {
        RRSetup R;
        rr_setup(t, S, p, sync, R);
        if (S == 1) {
          T = umax(rr_single_stage(R), R.Tsync);
        } else if (umax(rr_lower(R), R.Tsync) <= theta) {
          u64 t_lo, t_hi;
          const int rc = rr_sim(R, q.rounds ? q.rounds : RR_SIM_ROUNDS, theta, t_lo, t_hi, nullptr);
          if (rc == RR_MET || (rc == RR_BUDGET && R.Tsync >= t_hi)) {
            T = umax(t_lo, R.Tsync);
          } else if (rc == RR_BUDGET && umax(t_lo, R.Tsync) <= theta) {
            const u32 k = atomicAdd(q.n, 1u);
            if (k < q.cap) {
              q.buf[3 * (u64)k] = i;
              q.buf[3 * (u64)k + 1] = t_lo;
              q.buf[3 * (u64)k + 2] = t_hi;
            } else {
              T = umax(rr_ceil_bf(R, t_lo, t_hi), R.Tsync);
            }
          }
        }
      }
      if (T < bestT) {  // indices increase along the chunk: strict < keeps the first
        bestT = T;
        bestI = i;
        if (T < gb) atomicMin((unsigned long long *)&rs->best, T);
      }
      ++cnt;
      if (i + 1 == i1) break;
      if (!SP::next(cuts, S - 1, sp.L - 1)) {  // cut set exhausted: next composition
        cuts = first_subset<PK>(S - 1);
        if (!SP::next(Rp, comp_k(sp, S), comp_n(sp))) {  // compositions exhausted: next S
          ++S;
          if (S > sp.s_max) break;
          Rp = first_subset<PK>(comp_k(sp, S));
          cuts = first_subset<PK>(S - 1);
        }
      }
    }
  }
  block_minloc_store<RR_NT>(bestT, bestI, cnt, out + blockIdx.x);
}

// The deferred candidates of k_search_rr that can still win (bracket low <= the launch's best; a tie
// may win on its index), a warp each; one (T, index) per block into out (count 0: the search kernel
// counted them).
__global__ void __launch_bounds__(RR_NT) k_rr_drain_search(DevTables g, SearchSpace sp, BlockOut *out, ModelP m,
                                                           const RRSearchSched *rs, RRQueue q) {
  const u32 n = umin(*q.n, q.cap);
  u64 bestT = U64MAX, bestI = U64MAX;
  if (n > 0) {
    typedef SpaceT<P8> SP;
    typedef typename SP::PK PK;
    constexpr int BK = SP::BK;
    extern __shared__ u64 sm[];
    __shared__ long long dist[RR_NT / 32][RR_BF_NODES];
    u64 *Bn = sm + smem_words(g.L, g.N);
    const int nb = ((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK;
    for (int i = threadIdx.x; i < nb; i += RR_NT) Bn[i] = g_binom[i / BK][i % BK];
    const SmemTab t = stage_tables<false>(g, sm);
    const u64 best = rs->best;
    const int w = threadIdx.x >> 5;
    for (u32 k = blockIdx.x * (RR_NT / 32) + w; k < n; k += gridDim.x * (RR_NT / 32)) {
      const u64 i = q.buf[3 * (u64)k], t_lo = q.buf[3 * (u64)k + 1], t_hi = q.buf[3 * (u64)k + 2];
      if (t_lo > best) continue;  // warp-uniform
      int S;
      PK Rp, cuts;
      unrank_global_smem<BK>(sp, i, S, Rp, cuts, Bn);
      const P8 p = part_from<P8>(sp, S, Rp, cuts);
      RRSetup R;
      rr_setup(t, S, p, (int)m.sync, R);
      const u64 T = umax(rr_ceil_bf_warp(R, t_lo, t_hi, dist[w]), R.Tsync);
      if (better(T, i, bestT, bestI)) bestT = T, bestI = i;
    }
  }
  block_minloc_store<RR_NT>(bestT, bestI, 0, out + blockIdx.x);
}

int launch_search_rr(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, const ModelP &m, int sms,
                     BlockOut *out, int max_blocks, int *nblocks, void *sched, const RRQueue &q, cudaStream_t st) {
  static_assert(sizeof(RRSearchSched) <= SEARCH_SCHED_BYTES, "schedule slot");
  const u64 span = end - begin;
  const size_t smem = ((size_t)smem_words(g.L, g.N) +
                       (size_t)(((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK8)) * sizeof(u64);
  static bool attr = false;
  if (!attr) {
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, k_rr_drain_search);
    cudaFuncSetAttribute(k_rr_drain_search, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         227 * 1024 - (int)fa.sharedSizeBytes);
    attr = true;
  }
  u64 wave = (u64)sms * 2;
  if (wave > (u64)max_blocks / 2) wave = (u64)max_blocks / 2;
  u64 chunk = span / (wave * RR_NT * 8);
  if (chunk < 1) chunk = 1;
  while ((span + chunk - 1) / chunk >= (1ull << 31)) chunk *= 2;
  u64 blocks = ((span + chunk - 1) / chunk + RR_NT - 1) / RR_NT;
  if (blocks > wave) blocks = wave;
  if (blocks == 0) blocks = 1;
  u64 dblocks = (u64)sms < (u64)max_blocks - blocks ? (u64)sms : (u64)max_blocks - blocks;
  RRSearchSched *rs = (RRSearchSched *)sched;
  cudaMemsetAsync(rs, 0, sizeof(RRSearchSched), st);
  cudaMemsetAsync(&rs->best, 0xFF, sizeof(u64), st);
  cudaMemsetAsync(q.n, 0, sizeof(u32), st);
  k_search_rr<<<(unsigned)blocks, RR_NT, smem, st>>>(g, sp, begin, end, chunk, out, m, rs, q);
  k_rr_drain_search<<<(unsigned)dblocks, RR_NT, smem, st>>>(g, sp, out + blocks, m, rs, q);
  *nblocks = (int)(blocks + dblocks);
  return 2;
}

int launch_search_generic(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, int path32, const ModelP &m,
                          bool wide, int sms, BlockOut *out, int max_blocks, int *nblocks, void *sched,
                          cudaStream_t st, bool dense) {
  constexpr int NT = 256;
  const u64 span = end - begin;
#ifndef DENSE_DFS
#define DENSE_DFS 0  // 1: small spaces through one threshold-walk launch (B200: C2 0.27 -> 0.23 ms, GNMT 0.11 -> 0.20 ms)
#endif
  if (dense && DENSE_DFS && m.sched == SCHED_PIPEDREAM) {
    // a small space in one launch of the threshold walk: one wave, chunks of about span / threads
    const bool both = path32 < 0;
    const u64 room = both ? (u64)max_blocks / 2 : (u64)max_blocks;
    const u64 wave = (u64)sms * DFS_MINB < room ? (u64)sms * DFS_MINB : room;
    u64 chunk = (span + wave * NT - 1) / (wave * NT);
    if (chunk < 1) chunk = 1;
    u64 blocks = ((span + chunk - 1) / chunk + NT - 1) / NT;
    if (blocks > wave) blocks = wave;
    if (blocks == 0) blocks = 1;
    const int BK = wide ? BINOM_K : BK8;
    const size_t smem = ((size_t)smem_words(g.L, g.N) +
                         (size_t)(((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK)) * sizeof(u64);
    const int p32 = path32 >= 0 ? (path32 & 1) : path32;
    if (wide) run_search_generic<NT, P16>((unsigned)blocks, smem, st, g, sp, begin, end, chunk, out, m, p32, sched);
    else run_search_generic<NT, P8>((unsigned)blocks, smem, st, g, sp, begin, end, chunk, out, m, p32, sched);
    *nblocks = (int)blocks * (both ? 2 : 1);
    return both ? 2 : 1;
  }
  if (dense) {
    // a small space in one launch, latency first: every candidate scored exactly by its own thread
    // (or two), as many blocks as the result area holds
    const bool both = path32 < 0 && m.sched == SCHED_PIPEDREAM;
    const u64 room = both ? (u64)max_blocks / 2 : (u64)max_blocks;
    u64 per = (span + room * NT - 1) / (room * NT);
    if (per == 0) per = 1;
    u64 blocks = (span + per * NT - 1) / (per * NT);
    if (blocks == 0) blocks = 1;
    const int BK = wide ? BINOM_K : BK8;
    const size_t smem = ((size_t)smem_words(g.L, g.N, true) +
                         (size_t)(((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK)) * sizeof(u64);
    ModelP mm = m;
    const unsigned nbk = (unsigned)blocks;
#define DENSE_LAUNCH(PT)                                                                                  \
  if (m.sched != SCHED_PIPEDREAM) run_search_generic<NT, PT>(nbk, smem, st, g, sp, begin, end, per, out, mm, path32 & 1, sched); \
  else if (path32 == 3) k_search_generic<NT, true, SCHED_PIPEDREAM, PT, true><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out, mm, -1); \
  else if (path32 == 2) k_search_generic<NT, false, SCHED_PIPEDREAM, PT, true><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out, mm, -1); \
  else if (path32 == 1) k_search_generic<NT, true, SCHED_PIPEDREAM, PT><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out, mm, -1); \
  else if (path32 == 0) k_search_generic<NT, false, SCHED_PIPEDREAM, PT><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out, mm, -1); \
  else {                                                                                                  \
    k_search_generic<NT, true, SCHED_PIPEDREAM, PT><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out, mm, 1); \
    k_search_generic<NT, false, SCHED_PIPEDREAM, PT><<<nbk, NT, smem, st>>>(g, sp, begin, end, per, out + nbk, mm, 0); \
  }
    if (wide) { DENSE_LAUNCH(P16) } else { DENSE_LAUNCH(P8) }
#undef DENSE_LAUNCH
    *nblocks = (int)blocks * (both ? 2 : 1);
    return both ? 2 : 1;
  }
  // at least 4 candidates per thread (the unrank is a few binary searches); up to 8 blocks per SM.
  // A flushed schedule costs ~M S stage steps per candidate: one candidate per thread is enough.
  // A small span (a launch of a short model's space) is latency-bound: one candidate per thread.
  // The pruned schedules (GPipe, DAPPLE, Chimera): one candidate per thread still measured fastest
  // (B200, BERT-24 M = 8, per-thread counts 1 / 4 / 16 / 64: GPipe 2.97 / 2.88 / 3.84 / 7.3 ms,
  // DAPPLE 4.12 / 4.10 / 5.03 / 6.7, Chimera 11.3 / 10.9 / 19.9 / 50.1): about a third of the
  // candidates survive the bound, and their full recurrences want every thread.
#ifndef PRUNE_PER
#define PRUNE_PER 1
#endif
  const bool pruned = m.sched == SCHED_GPIPE || m.sched == SCHED_DAPPLE || m.sched == SCHED_CHIMERA;
  const u64 min_per = pruned ? (u64)PRUNE_PER
                      : (m.sched == SCHED_RR || span <= (u64)sms * 8 * NT * 4) ? 1 : 4;
  u64 threads = (span + min_per - 1) / min_per;
  u64 blocks = (threads + NT - 1) / NT;
  const bool both = path32 < 0 && m.sched == SCHED_PIPEDREAM;  // two gated launches share max_blocks
  const u64 room = both ? (u64)max_blocks / 2 : (u64)max_blocks;
  const u64 cap = (u64)sms * 8 < room ? (u64)sms * 8 : room;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  u64 per = (span + blocks * NT - 1) / (blocks * NT);
  if (m.sched == SCHED_PIPEDREAM) {
    // the threshold walk: one wave of resident blocks drawing chunks of about span / (8 x threads)
    // candidates (at least DFS_MINCH) from the launch's counter
    const u64 wave = (u64)sms * DFS_MINB < room ? (u64)sms * DFS_MINB : room;
    u64 chunk = span / (wave * NT * 8);
    if (chunk < (u64)DFS_MINCH) chunk = DFS_MINCH;
    while ((span + chunk - 1) / chunk >= (1ull << 31)) chunk *= 2;
    const u64 nch = (span + chunk - 1) / chunk;
    blocks = (nch + NT - 1) / NT;
    if (blocks > wave) blocks = wave;
    if (blocks == 0) blocks = 1;
    per = chunk;
  }
  const int BK = wide ? BINOM_K : BK8;
  const size_t smem = ((size_t)smem_words(g.L, g.N) +
                       (size_t)(((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK)) * sizeof(u64);
  const unsigned nbk = (unsigned)blocks;
  const u64 pt = per ? per : 1;
  if (wide) run_search_generic<NT, P16>(nbk, smem, st, g, sp, begin, end, pt, out, m, path32, sched);
  else run_search_generic<NT, P8>(nbk, smem, st, g, sp, begin, end, pt, out, m, path32, sched);
  *nblocks = (int)blocks * (both ? 2 : 1);
  return both ? 2 : 1;
}

// ---------------------------------------------------------------------------------------------
// grid-level finalisation: one block reduces the per-block (T, index, count) entries, then decodes
// the winning index into its partition record (16 bytes, or 32 for a wide space).
// ---------------------------------------------------------------------------------------------
// res: the ResultDev layout (time_ns, index, evaluated, record) with the record cut to rec_bytes (16 or
// 32), so it can be the caller's autopipe_result / autopipe_result_w directly (asynchronous search)
__global__ void __launch_bounds__(256) k_finalize(const BlockOut *in, int n, SearchSpace sp, ResultDev *res, int wide,
                                                 int rec_bytes) {
  // binomial rows 0..L (all the unranking needs) in shared memory: the winner is decoded with
  // fixed-length binary searches instead of a serial walk over __constant__ (which misses its cache)
  __shared__ u64 Bn[(MAXL + 1) * BINOM_K];
  const int BK = wide ? BINOM_K : BK8;
  const int rows = (sp.L > sp.N ? sp.L : sp.N) + 1;  // cut sets of {0..L-2}, compositions of {1..N}
  for (int i = threadIdx.x; i < rows * BK; i += 256) Bn[i] = g_binom[i / BK][i % BK];
  u64 t = U64MAX, idx = U64MAX, cnt = 0;
  for (int i = threadIdx.x; i < n; i += 256) {
    const BlockOut b = in[i];
    if (better(b.t, b.idx, t, idx)) { t = b.t; idx = b.idx; }
    cnt += b.count;
  }
  __shared__ BlockOut slot;
  block_minloc_store<256>(t, idx, cnt, &slot);
  __syncthreads();
  if (threadIdx.x == 0) {
    res->time_ns = slot.t;
    res->index = slot.idx;
    res->evaluated = slot.count;
    unsigned char rec[32];
    for (int i = 0; i < 32; ++i) rec[i] = 0xFF;
    const int off = wide ? 16 : 8;
    if (slot.idx != U64MAX) {
      int S;
      if (wide) {
        Pk2 Rp, cuts;
        unrank_global_smem<BINOM_K>(sp, slot.idx, S, Rp, cuts, Bn);
        const P16 p = part_from<P16>(sp, S, Rp, cuts);
        rec[0] = (unsigned char)S;
        for (int s = 0; s < S - 1; ++s) rec[1 + s] = (unsigned char)p.cut(s);
        for (int s = 0; s < S; ++s)
          for (int w = 0; w < MAXNW; ++w)
            if ((p.mask(s) >> w) & 1) rec[off + w] = (unsigned char)s;
      } else {
        u64 Rp, cuts;
        unrank_global_smem<BK8>(sp, slot.idx, S, Rp, cuts, Bn);
        const P8 p = part_from<P8>(sp, S, Rp, cuts);
        rec[0] = (unsigned char)S;
        for (int s = 0; s < S - 1; ++s) rec[1 + s] = (unsigned char)p.cut(s);
        for (int s = 0; s < S; ++s)
          for (int w = 0; w < MAXN; ++w)
            if ((p.mask(s) >> w) & 1) rec[off + w] = (unsigned char)s;
      }
    }
    for (int i = 0; i < rec_bytes; ++i) res->part[i] = rec[i];
  }
}

int launch_finalize(const BlockOut *in, int n, const SearchSpace &sp, ResultDev *out, bool wide, cudaStream_t st,
                    int rec_bytes) {
  k_finalize<<<1, 256, 0, st>>>(in, n, sp, out, wide ? 1 : 0, rec_bytes);
  return 1;
}

// Row e (multi-GPU): the per-rank search results gathered into one array (an all-gather of
// autopipe_result bytes) reduced to their lexicographic (time_ns, index) minimum, evaluated counts
// summed, the winner's record copied. One warp; n is the number of ranks.
__global__ void k_reduce_results(const unsigned char *in, unsigned n, int rec_bytes, unsigned char *out) {
  const unsigned stride = 24u + (unsigned)rec_bytes;
  u64 t = U64MAX, idx = U64MAX, cnt = 0;
  unsigned who = 0xFFFFFFFFu;
  for (unsigned i = threadIdx.x; i < n; i += 32) {
    const u64 *r = (const u64 *)(in + (size_t)i * stride);
    if (who == 0xFFFFFFFFu || better(r[0], r[1], t, idx)) {  // ascending i: the first of equals stays
      t = r[0];
      idx = r[1];
      who = i;
    }
    cnt += r[2];
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const u64 t2 = __shfl_xor_sync(0xffffffffu, t, o), i2 = __shfl_xor_sync(0xffffffffu, idx, o);
    const unsigned w2 = __shfl_xor_sync(0xffffffffu, who, o);
    // ties on (t, idx) (empty results: both UINT64_MAX) resolve to the lower rank, so the copied record
    // is deterministic
    if (better(t2, i2, t, idx) || (t2 == t && i2 == idx && w2 < who)) { t = t2; idx = i2; who = w2; }
    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  }
  if (threadIdx.x == 0) {
    u64 *o = (u64 *)out;
    o[0] = t;
    o[1] = idx;
    o[2] = cnt;
    const unsigned char *src = in + (size_t)(who == 0xFFFFFFFFu ? 0 : who) * stride + 24;
    for (int b = 0; b < rec_bytes; ++b) out[24 + b] = (n == 0) ? (unsigned char)0xFF : src[b];
  }
}

int launch_reduce_results(const void *in, unsigned n, int rec_bytes, void *out, cudaStream_t st) {
  k_reduce_results<<<1, 32, 0, st>>>((const unsigned char *)in, n, rec_bytes, (unsigned char *)out);
  return 1;
}

void upload_binomials_search(const u64 (*tab)[BINOM_K]) { upload_binomials_tu(tab); }

}  // namespace ap
