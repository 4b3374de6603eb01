// k_search_r1.cu — the hot kernel: exhaustive search over the block of the space in which every
// stage runs on one worker (composition R = 1..S, rho = 0 in SPEC.md §5). For the 96-layer, 8-stage
// workload this block IS the space: C(95,7) = 11,050,084,695 cut sets (rows a3-a8).
//
// What each candidate costs. With r = 1 the closed form of SPEC.md §4 is
//   T = max( c_s, lm_s, ceil(W(s,t) / (t-s+1)) ),  W(s,t) = sum_{u=s..t} c_u + sum_{u=s..t-1} z_u,
// (c_s = stage cost on its worker, z_s = cf_s + cb_s, lm_s = max(cf_s, cb_s)). The search only needs,
// per candidate, the exact decision "T <= theta" against the running best (theta = best or best-1),
// and T <= theta iff every term <= theta, i.e. W(s,t) <= theta*(t-s+1) — no division. With the cut
// sets ordered (outer cuts, x = e_{S-3}, e = e_{S-2}), the terms that involve the last cut e collapse
// into three comparisons against per-row thresholds:
//   A[e] <= H1,  K[e] <= H2,  V[e] <= theta,
// where A[e] = PC_p[e+1], K[e] = PC_p[e+1] + Z_p[e] + (PC_q[L] - PC_q[e+1]), V[e] = max(c_q, lm_p) are
// per-state column tables (p = S-2, q = S-1), and H1, H2 fold every other term of the candidate.
// A candidate that passes gets its exact T (with the divisions) and index; it is the rare path.
// Every candidate of the shard is decided individually; none is skipped.
//
// Mapping (the B200 part). Work is grouped by x: all rows (outer cut tuples below x) with the same x
// have the same number of columns l = L-2-x, so a warp takes 32 rows of one x (one per lane, R
// consecutive rows per lane) and sweeps the columns in lockstep: the column tables are read with
// broadcast LDS.128 (one shared-memory wavefront per warp step), per-lane thresholds stay in
// registers, and there is no divergence in the hot loop. Consecutive rows of a lane differ in one
// cut (lexicographic successor), so the per-row threshold update touches two stages; a full
// re-hoist happens only when an earlier cut changes. Warps take tasks from a global atomic counter
// (persistent grid, a few blocks per SM); the (T, index) argmin is per lane, then warp -> block
// (shuffles + shared memory) -> grid (k_finalize). The result is the lexicographic (T, index)
// minimum, independent of the task order, the grid size and the number of GPUs.
#include "binom.cuh"
#include "internal.h"

namespace ap {

struct R1XEntry {      // one x value of the schedule (host-built, SPEC.md §5 shard arithmetic)
  int x;               // e_{S-3}
  u32 rows_per_lane;   // R
  u64 row_begin;       // first row (lex rank of the outer tuple among NO-subsets of {0..x-1})
  u64 row_end;         // one past the last row in the shard
  u64 task_begin;      // global index of this x's first task
};

struct R1Header {
  u64 off;                    // global index of (S, rho = 0, kappa = 0)
  u64 ntasks;
  u64 lo_outer, hi_outer;     // packed outer cuts of the shard's first / last candidate
  int lo_x, lo_e, hi_x, hi_e; // their x and e
  int nx, pad;
  u32 counter;                // task counter (reset per launch)
  u32 pad2;
};

template <typename T>
struct __align__(16) ColT {
  T A, K, V, pad;
};
template <typename T>
struct __align__(16) RowT {
  T PCa, PCb, Z, LM;  // PC_{p-2}[y+1], PC_{p-1}[y+1], Z_{p-2}[y], LM_{p-2}[y]
};

typedef long long i64;
// theta >= THETA_ALL means "no best yet": every candidate passes (all modelled times are < 2^59,
// so theta * 8 never overflows i64 for a real theta)
constexpr i64 THETA_ALL = 1ll << 60;

__device__ __forceinline__ i64 smin(i64 a, i64 b) { return a < b ? a : b; }

// exact T of an r = 1 candidate (all divisions), from the u64 tables in shared memory
template <int S>
__device__ __noinline__ u64 exact_T_r1(const u64 *PC, const u64 *Z, const u64 *LM, int L, u64 cuts) {
  const int Lp1 = L + 1;
  u64 c[S], z[S];
  u64 T = 0;
#pragma unroll
  for (int s = 0; s < S; ++s) {
    const int a = (s == 0) ? 0 : byte_at(cuts, s - 1) + 1;
    const int e = (s == S - 1) ? L - 1 : byte_at(cuts, s);
    c[s] = PC[s * Lp1 + e + 1] - PC[s * Lp1 + a];
    T = umax(T, c[s]);
    z[s] = 0;
    if (s < S - 1) {
      z[s] = Z[s * L + e];
      T = umax(T, LM[s * L + e]);
    }
  }
#pragma unroll
  for (int s = 0; s < S - 1; ++s) {
    u64 acc = c[s];
#pragma unroll
    for (int t = s + 1; t < S; ++t) {
      acc += z[t - 1] + c[t];
      T = umax(T, (acc + (u64)(t - s)) / (u64)(t - s + 1));
    }
  }
  return T;
}

// Per-lane search state for one S.
template <int S, typename T>
struct Lane {
  static constexpr int p = S - 2, q = S - 1, NO = S - 3;
  // level A (cuts e_0..e_{p-3}, stages 0..p-3)
  bool aliveA;
  i64 Ga, Gb, Gc, Gd;
  u64 baseA;  // PC_{p-2}[a_{p-2}]
  // task (x) level
  int x;
  u64 cx;      // PC_{p-1}[x+1] (S >= 4) or the stage-0 cost (S = 3)
  u64 zx, lmx; // Z_{p-1}[x], LM_{p-1}[x]
  u64 base_p;  // PC_p[x+1]
  // row
  u64 outer;   // packed e_0..e_{NO-1}
  bool alive;
  T H1, H2, TH;
  // best
  u64 bestT, bestI;
  i64 theta;
};

template <int S, typename T>
__device__ __forceinline__ void hoist_A(Lane<S, T> &st, const u64 *PC, const u64 *Z, const u64 *LM, int L) {
  constexpr int p = S - 2;
  const int Lp1 = L + 1;
  const i64 th = st.theta;
  bool ok = true;
  i64 Ga = THETA_ALL * 4, Gb = THETA_ALL * 4, Gc = THETA_ALL * 4, Gd = THETA_ALL * 4;
  u64 baseA = 0;
  if constexpr (p >= 3) {
    const int a2 = byte_at(st.outer, p - 3) + 1;
    baseA = PC[(p - 2) * Lp1 + a2];
  }
  if (th >= THETA_ALL) {
    st.aliveA = true;
    st.Ga = Ga; st.Gb = Gb; st.Gc = Gc; st.Gd = Gd;
    st.baseA = baseA;
    return;
  }
  if constexpr (p >= 3) {
    // stages 0..p-3 are fixed by the cuts e_0..e_{p-3}
    i64 c[p - 2 > 0 ? p - 2 : 1], z[p - 2 > 0 ? p - 2 : 1];
#pragma unroll
    for (int u = 0; u <= p - 3; ++u) {
      const int a = (u == 0) ? 0 : byte_at(st.outer, u - 1) + 1;
      const int e = byte_at(st.outer, u);
      c[u] = (i64)(PC[u * Lp1 + e + 1] - PC[u * Lp1 + a]);
      z[u] = (i64)Z[u * L + e];
      ok &= (c[u] <= th) & ((i64)LM[u * L + e] <= th);
    }
    // segments inside stages 0..p-3
#pragma unroll
    for (int s = 0; s <= p - 3; ++s) {
      i64 acc = c[s];
#pragma unroll
      for (int t = s + 1; t <= p - 3; ++t) {
        acc += z[t - 1] + c[t];
        ok &= acc <= th * (t - s + 1);
      }
    }
    // D'_s = sum_{u=s}^{p-3} (c_u + z_u) and the four collapsed thresholds
    i64 D = 0;
#pragma unroll
    for (int s = p - 3; s >= 0; --s) {
      D += c[s] + z[s];
      Ga = smin(Ga, th * (p - 1 - s) - D);
      Gb = smin(Gb, th * (p - s) - D);
      Gc = smin(Gc, th * (p - s + 1) - D);
      Gd = smin(Gd, th * (p - s + 2) - D);
    }
  }
  st.aliveA = ok;
  st.Ga = Ga; st.Gb = Gb; st.Gc = Gc; st.Gd = Gd;
  st.baseA = baseA;
}

template <typename T>
__device__ __forceinline__ T clampT(i64 v) {
  // threshold for "value <= v" on values of type T (< 2^32 - 16 in the 32-bit path)
  if (v < 0) return (T)0;  // caller folds the "dead" case separately
  const u64 m = (sizeof(T) == 4) ? 0xFFFFFFFFull : ~0ull;
  return (T)((u64)v > m ? m : (u64)v);
}

// Row thresholds for the current (outer, x) with the current theta.
template <int S, typename T>
__device__ __forceinline__ void hoist_row(Lane<S, T> &st, const RowT<T> *rowy) {
  constexpr int p = S - 2;
  const i64 th = st.theta;
  if (th >= THETA_ALL) {
    st.alive = true;
    st.H1 = st.H2 = st.TH = (T)~(T)0;
    return;
  }
  i64 h1, h2;
  bool ok = st.aliveA;
  if constexpr (S == 3) {
    const i64 c0 = (i64)st.cx, zx = (i64)st.zx;
    ok &= (c0 <= th) & ((i64)st.lmx <= th);
    h1 = smin(th, 2 * th - c0 - zx);
    h2 = smin(2 * th, 3 * th - c0 - zx);
  } else {
    const int y = byte_at(st.outer, S - 4);  // e_{p-2}
    const RowT<T> r = rowy[y];
    const i64 cpm2 = (i64)((u64)r.PCa - st.baseA);
    const i64 cpm1 = (i64)(st.cx - (u64)r.PCb);
    const i64 zpm2 = (i64)(u64)r.Z;
    const i64 Q = cpm2 + zpm2 + cpm1;
    const i64 zx = (i64)st.zx;
    ok &= (cpm2 <= smin(th, st.Ga)) & ((i64)(u64)r.LM <= th) & (cpm1 <= th) & (Q <= smin(2 * th, st.Gb)) &
          ((i64)st.lmx <= th);
    h1 = smin(smin(th, 2 * th - cpm1 - zx), smin(3 * th, st.Gc) - Q - zx);
    h2 = smin(smin(2 * th, 3 * th - cpm1 - zx), smin(4 * th, st.Gd) - Q - zx);
    (void)p;
  }
  const i64 H1 = h1 + (i64)st.base_p, H2 = h2 + (i64)st.base_p;
  ok &= (h1 >= 0) & (h2 >= 0);
  st.alive = ok;
  // dead rows: thresholds that no value can meet (values are >= 0, compare with <=): use H < 0 ->
  // encode by alive flag folded into TH (TH = 0 with alive = false never matters: we test alive).
  st.H1 = clampT<T>(H1);
  st.H2 = clampT<T>(H2);
  st.TH = clampT<T>(th);
}

template <int S, typename T, int NT>
__global__ void __launch_bounds__(NT) k_search_r1(DevTables g, const R1Header *__restrict__ hdr_g,
                                                  const R1XEntry *__restrict__ xt_g, R1Header *counter_hdr,
                                                  BlockOut *out) {
  constexpr int p = S - 2, q = S - 1, NO = S - 3;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int L = (int)g.L, Lp1 = L + 1, n = L - 1;
  __shared__ R1Header hdr;
  if (threadIdx.x == 0) hdr = *hdr_g;
  // shared layout: col[n] | rowy[n] | PC[S][Lp1] | Z[S-1][L] | LM[S-1][L] | xt[nx]
  ColT<T> *col = (ColT<T> *)smraw;
  RowT<T> *rowy = (RowT<T> *)(col + n);
  u64 *PC = (u64 *)(rowy + n);
  u64 *Z = PC + S * Lp1;
  u64 *LM = Z + (S - 1) * L;
  R1XEntry *xt = (R1XEntry *)(LM + (S - 1) * L);
  for (int i = threadIdx.x; i < S * Lp1; i += NT) PC[i] = g.PC[i];
  for (int i = threadIdx.x; i < (S - 1) * L; i += NT) {
    Z[i] = g.Z[i];
    LM[i] = g.LM[i];
  }
  __syncthreads();
  const int nx = hdr.nx;
  for (int i = threadIdx.x; i < nx; i += NT) xt[i] = xt_g[i];
  for (int e = threadIdx.x; e < n; e += NT) {  // column tables (per state, per S)
    const u64 A = PC[p * Lp1 + e + 1];
    const u64 cq = PC[q * Lp1 + L] - PC[q * Lp1 + e + 1];
    ColT<T> cl;
    cl.A = (T)A;
    cl.K = (T)(A + Z[p * L + e] + cq);
    cl.V = (T)umax(cq, LM[p * L + e]);
    cl.pad = 0;
    col[e] = cl;
    RowT<T> rw;
    if constexpr (S >= 4) {
      rw.PCa = (T)PC[(p - 2) * Lp1 + e + 1];
      rw.Z = (T)Z[(p - 2) * L + e];
      rw.LM = (T)LM[(p - 2) * L + e];
    } else {
      rw.PCa = 0; rw.Z = 0; rw.LM = 0;
    }
    rw.PCb = (T)PC[(p - 1) * Lp1 + e + 1];
    rowy[e] = rw;
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  Lane<S, T> st;
  st.bestT = U64MAX;
  st.bestI = U64MAX;
  u64 cnt = 0;
  const u64 ntasks = hdr.ntasks;
  for (;;) {
    u64 task = 0;
    if (lane == 0) task = atomicAdd(&counter_hdr->counter, 1u);
    task = __shfl_sync(0xffffffffu, task, 0);
    if (task >= ntasks) break;
    // locate the x entry (entries are few; linear scan over shared memory, warp-uniform)
    int xi = 0;
    while (xi + 1 < nx && xt[xi + 1].task_begin <= task) ++xi;
    const R1XEntry xe = xt[xi];
    const int x = xe.x;
    const u64 R = xe.rows_per_lane;
    const u64 r0 = xe.row_begin + (task - xe.task_begin) * 32ull * R + (u64)lane * R;
    const u64 r1 = umin(r0 + R, xe.row_end);
    // task-level values
    st.x = x;
    if constexpr (S == 3) {
      st.cx = PC[0 * Lp1 + x + 1];
      st.zx = Z[0 * L + x];
      st.lmx = LM[0 * L + x];
    } else {
      st.cx = PC[(p - 1) * Lp1 + x + 1];
      st.zx = Z[(p - 1) * L + x];
      st.lmx = LM[(p - 1) * L + x];
    }
    st.base_p = PC[p * Lp1 + x + 1];
    const bool has_rows = r0 < r1;
    const int e_first = x + 1, e_last = L - 2;
    if (has_rows) {
      // lex unrank of the lane's first row among NO-subsets of {0..x-1}
      st.outer = (NO > 0) ? lex_unrank_packed(r0, NO, x) : 0ull;
    } else {
      st.outer = 0;
    }
    // the theta used for filtering: T <= theta passes. Non-strict (theta = best) while a candidate
    // of this task may still have a smaller index than the lane's best, strict (best - 1) once the
    // lane's candidates are past it (indices increase along a lane's rows and columns).
    bool strict = true;
    if (has_rows && st.bestT != U64MAX) {
      int e0 = e_first;
      if (st.outer == hdr.lo_outer && x == hdr.lo_x) e0 = hdr.lo_e > e0 ? hdr.lo_e : e0;
      const u64 first_idx =
          hdr.off + lex_rank_packed(st.outer | ((u64)x << (8 * NO)) | ((u64)e0 << (8 * (NO + 1))), S - 1, n);
      strict = first_idx > st.bestI;
    }
    st.theta = (st.bestT == U64MAX) ? THETA_ALL : (i64)st.bestT - (strict ? 1 : 0);
    u64 row = r0;
    bool need_A = true;
    while (true) {
      const bool active = has_rows && row < r1;
      if (!__any_sync(0xffffffffu, active)) break;
      int emin = e_first, emax = e_last;
      u64 cuts_prefix = 0;  // outer cuts + x, packed (the candidate's cuts without e)
      if (active) {
        cuts_prefix = st.outer | ((u64)x << (8 * NO));
        // shard boundaries: the shard's first / last row may be partial
        if (st.outer == hdr.lo_outer && x == hdr.lo_x) emin = hdr.lo_e > emin ? hdr.lo_e : emin;
        if (st.outer == hdr.hi_outer && x == hdr.hi_x) emax = hdr.hi_e < emax ? hdr.hi_e : emax;
        cnt += (emax >= emin) ? (u64)(emax - emin + 1) : 0ull;
        if (need_A) hoist_A<S, T>(st, PC, Z, LM, L);
        hoist_row<S, T>(st, rowy);
        st.alive &= emax >= emin;
      } else {
        st.alive = false;
      }
      // ---- hot loop: lockstep sweep of the columns e in (x, L-2] -----------------------------
      bool alive = st.alive;
      int e = e_first;
      auto pass = [&](const ColT<T> &c) { return (c.A <= st.H1) & (c.K <= st.H2) & (c.V <= st.TH); };
      while (e <= e_last) {
        // 4 columns per step, one broadcast 128-bit shared load each
        bool hit = false;
        if (e + 3 <= e_last) {
          const ColT<T> c0 = col[e], c1 = col[e + 1], c2 = col[e + 2], c3 = col[e + 3];
          hit = alive & (pass(c0) | pass(c1) | pass(c2) | pass(c3));
          if (!hit) { e += 4; continue; }
        } else {
          hit = alive & pass(col[e]);
          if (!hit) { e += 1; continue; }
        }
        // rare path: re-check the (up to 4) columns in order with the current thresholds
        const int stop = (e + 3 <= e_last) ? e + 3 : e;
        for (int ee = e; ee <= stop; ++ee) {
          if (!(alive && pass(col[ee]))) continue;
          if (ee < emin || ee > emax) continue;  // outside the shard (partial rows only)
          const u64 cuts = cuts_prefix | ((u64)ee << (8 * (NO + 1)));
          const u64 Tc = exact_T_r1<S>(PC, Z, LM, L, cuts);
          const u64 idx = hdr.off + lex_rank_packed(cuts, S - 1, n);
          if (better(Tc, idx, st.bestT, st.bestI)) {
            st.bestT = Tc;
            st.bestI = idx;
          }
          // every later candidate of this lane's task has a larger index: strict from here on
          const i64 th_new = (i64)st.bestT - 1;
          if (th_new != st.theta) {
            st.theta = th_new;
            hoist_A<S, T>(st, PC, Z, LM, L);
            hoist_row<S, T>(st, rowy);
            alive = st.alive && (emax >= emin);
          }
        }
        e = stop + 1;
      }
      if (!active) {
        row = r1;  // idle lane: keep sweeping in lockstep until every lane is done
        continue;
      }
      // ---- next row: lexicographic successor of the outer cuts below x --------------------
      ++row;
      need_A = false;
      if (row < r1) {
        if constexpr (NO == 0) {
          // one row per x
        } else {
          const int ylast = byte_at(st.outer, NO - 1);
          if (ylast < x - 1) {
            st.outer += 1ull << (8 * (NO - 1));  // only e_{p-2} moves: level A unchanged
          } else {
            lex_next_packed(st.outer, NO, x);
            need_A = true;
          }
        }
      }
    }
  }
  block_minloc_store<NT>(st.bestT, st.bestI, cnt, out + blockIdx.x);
}

// ------------------------------------------------------------------------------------------------
// host side: the task schedule (rows per x restricted to the shard) and the launch
// ------------------------------------------------------------------------------------------------
static u64 hb(int n, int k) {  // host binomial (n < 256, k <= 8); exact in u64
  if (k < 0 || n < 0 || k > n) return 0;
  u64 r = 1;
  for (int i = 1; i <= k; ++i) r = r * (u64)(n - k + i) / (u64)i;
  return r;
}

static void host_unrank(u64 rank, int k, int n, int *out) {
  int x = 0;
  for (int i = 0; i < k; ++i) {
    while (hb(n - 1 - x, k - 1 - i) <= rank) {
      rank -= hb(n - 1 - x, k - 1 - i);
      ++x;
    }
    out[i] = x++;
  }
}

// number of k-subsets of {0..x-1} lexicographically smaller than the increasing tuple t[0..k-1]
static u64 count_less(int x, int k, const int *t) {
  u64 cnt = 0;
  int prev = -1;
  for (int i = 0; i < k; ++i) {
    const int lim = t[i] < x ? t[i] : x;
    for (int v = prev + 1; v < lim; ++v) cnt += hb(x - 1 - v, k - 1 - i);
    if (t[i] >= x) return cnt;
    prev = t[i];
  }
  return cnt;
}

template <int S, typename T>
static int launch_r1_t(const DevTables &g, const SearchSpace &sp, u64 k_begin, u64 k_end, int sms,
                       BlockOut *out, int max_blocks, int *nblocks, void *work, size_t work_bytes,
                       cudaStream_t st) {
  constexpr int NO = S - 3, NT = 256;
  const int L = (int)g.L, n = L - 1, k = S - 1;
  int lo[8], hi[8];
  host_unrank(k_begin, k, n, lo);
  host_unrank(k_end - 1, k, n, hi);
  // header + x table in pinned-less host memory, copied into the device work area
  static thread_local unsigned char hbuf[sizeof(R1Header) + 256 * sizeof(R1XEntry)];
  R1Header *h = (R1Header *)hbuf;
  R1XEntry *xt = (R1XEntry *)(hbuf + sizeof(R1Header));
  memset(h, 0, sizeof(*h));
  h->off = sp.off[S];
  for (int i = 0; i < NO; ++i) {
    h->lo_outer |= (u64)lo[i] << (8 * i);
    h->hi_outer |= (u64)hi[i] << (8 * i);
  }
  h->lo_x = lo[NO]; h->lo_e = lo[NO + 1];
  h->hi_x = hi[NO]; h->hi_e = hi[NO + 1];
  int nx = 0;
  u64 tasks = 0;
  const u64 TARGET = 384;  // candidates per lane per task
  for (int x = NO; x <= L - 3; ++x) {
    const bool lo_fits = (NO == 0) || lo[NO - 1] < x;
    const bool hi_fits = (NO == 0) || hi[NO - 1] < x;
    const u64 rb = count_less(x, NO, lo) + ((lo_fits && x < lo[NO]) ? 1 : 0);
    const u64 re = count_less(x, NO, hi) + ((hi_fits && x <= hi[NO]) ? 1 : 0);
    if (re <= rb) continue;
    const u64 ell = (u64)(L - 2 - x);
    u64 R = (TARGET + ell - 1) / ell;
    const u64 rows = re - rb;
    // keep at least ~8 tasks per SM overall: do not make R larger than needed
    const u64 nt = (rows + 32 * R - 1) / (32 * R);
    R1XEntry &xe = xt[nx++];
    xe.x = x;
    xe.rows_per_lane = (u32)R;
    xe.row_begin = rb;
    xe.row_end = re;
    xe.task_begin = tasks;
    tasks += nt;
  }
  h->nx = nx;
  h->ntasks = tasks;
  *nblocks = 0;
  if (tasks == 0) return 0;
  const size_t hbytes = sizeof(R1Header) + (size_t)nx * sizeof(R1XEntry);
  // one 16 KB slot per S, so the r = 1 launches of one search never share a schedule buffer
  if ((size_t)(S + 1) * 16384 > work_bytes || hbytes > 16384) return 0;
  work = (unsigned char *)work + (size_t)S * 16384;
  // pageable source: the call returns once hbuf has been staged, so hbuf may be reused at once
  cudaMemcpyAsync(work, hbuf, hbytes, cudaMemcpyHostToDevice, st);
  const size_t smem = (size_t)n * (sizeof(ColT<T>) + sizeof(RowT<T>)) + (size_t)S * (L + 1) * 8 +
                      2 * (size_t)(S - 1) * L * 8 + (size_t)nx * sizeof(R1XEntry);
  cudaFuncSetAttribute(k_search_r1<S, T, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_search_r1<S, T, NT>, NT, smem);
  if (per_sm < 1) per_sm = 1;
  u64 blocks = (u64)sms * per_sm;
  const u64 need = (tasks + (NT / 32) - 1) / (NT / 32);
  if (blocks > need) blocks = need;
  if (blocks > (u64)max_blocks) blocks = (u64)max_blocks;
  const R1Header *hd = (const R1Header *)work;
  const R1XEntry *xd = (const R1XEntry *)((unsigned char *)work + sizeof(R1Header));
  k_search_r1<S, T, NT><<<(unsigned)blocks, NT, smem, st>>>(g, hd, xd, (R1Header *)work, out);
  *nblocks = (int)blocks;
  return 1;
}

template <typename T>
static int launch_r1_s(int S, const DevTables &g, const SearchSpace &sp, u64 a, u64 b, int sms, BlockOut *out,
                       int mb, int *nb, void *w, size_t wb, cudaStream_t st) {
  switch (S) {
    case 3: return launch_r1_t<3, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
    case 4: return launch_r1_t<4, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
    case 5: return launch_r1_t<5, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
    case 6: return launch_r1_t<6, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
    case 7: return launch_r1_t<7, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
    case 8: return launch_r1_t<8, T>(g, sp, a, b, sms, out, mb, nb, w, wb, st);
  }
  return 0;
}

int launch_search_r1(const DevTables &g, const SearchSpace &sp, int S, u64 k_begin, u64 k_end, int path32,
                     int sms, BlockOut *out, int max_blocks, int *nblocks, void *work, size_t work_bytes,
                     cudaStream_t st) {
  if (path32)
    return launch_r1_s<u32>(S, g, sp, k_begin, k_end, sms, out, max_blocks, nblocks, work, work_bytes, st);
  return launch_r1_s<u64>(S, g, sp, k_begin, k_end, sms, out, max_blocks, nblocks, work, work_bytes, st);
}

}  // namespace ap
