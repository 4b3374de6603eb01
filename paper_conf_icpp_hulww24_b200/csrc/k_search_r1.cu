// k_search_r1.cu — the hot kernel: exhaustive search over the block of the space in which every
// stage runs on one worker (composition R = 1..S, rho = 0 in SPEC.md §5), S in [5, 8]. For the
// 96-layer, 8-stage workload this block IS the space: C(95,7) = 11,050,084,695 cut sets
// (rows a3-a8). Smaller S (tiny spaces) go through the generic kernel.
//
// What each candidate costs. With r = 1 the closed form of SPEC.md §4 is
//   T = max( c_s, lm_s, ceil(W(s,t) / (t-s+1)) ),  W(s,t) = sum_{u=s..t} c_u + sum_{u=s..t-1} z_u
// (c_s = stage cost on its worker, z_s = cf_s + cb_s, lm_s = max(cf_s, cb_s) at cut e_s). The search
// only needs, per candidate, the exact decision "T <= theta" against the running best (theta = best,
// or best - 1 once the lane is past the best's index), and T <= theta iff every term <= theta, i.e.
// W(s,t) <= theta * (t-s+1): no division. Scanning the stages left to right with
//   M_j(k) = min_{s<=j} ( theta * (j-s+1+k) - sum_{u=s..j} (c_u + z_u) ),
//   M_j(k) = min(theta * (1+k), M_{j-1}(k+1)) - (c_j + z_j),
// every segment that ends k stages after stage j is "rest <= M_j(k)". For the last two stages
// p = S-2 (layers x+1..e) and q = S-1 (layers e+1..L-1) all terms collapse into three comparisons
//   A[e] < H1',  K[e] < H2',  V[e] < TH',
// with per-state column tables A[e] = PC_p[e+1], K[e] = PC_p[e+1] + Z_p[e] + (PC_q[L] - PC_q[e+1]),
// V[e] = max(c_q, lm_p), and per-lane thresholds H1 = min(theta, M_{p-1}(1)) + PC_p[x+1],
// H2 = min(2 theta, M_{p-1}(2)) + PC_p[x+1], TH = theta (the ' versions are +1 for a strict test,
// and 0 for a lane whose fixed terms already exceed theta). A candidate that passes gets its exact T
// (with the divisions) and its index: the rare path. Every candidate of the shard is decided.
//
// Mapping (the B200 part). Cut sets are (prefix e_0..e_{S-5}, y = e_{S-4}, x = e_{S-3}, e = e_{S-2}).
// A warp task fixes y; its 32 lanes take different prefixes (R consecutive ones each). So within a
// warp, x and e run in lockstep and everything that depends on x or e only is warp-uniform: the
// x-level update is a broadcast load plus ~20 integer ops per lane, the column sweep reads a
// warp-private folded table with broadcast 128-bit shared-memory loads (8 columns, two x values,
// one compare of their minimum per step on the 32-bit path), and there is no divergence in the hot
// loop. A lane re-derives its prefix terms (O(S^2)) once per row; a row covers
// C(L-2-y, 2) candidates. Warps take tasks from a global atomic counter (persistent grid); the
// (T, index) argmin goes lane -> warp -> block (shuffles + shared memory) -> grid (k_finalize), so the
// result is the lexicographic (T, index) minimum whatever the task order, grid or GPU count.
#include <cstdlib>

#include "binom.cuh"
#include "internal.h"

namespace ap {

constexpr int R1_MAXCHUNK = 16;
// x values per pass of the column sweep, per path (B200: 2 for the 32-bit tables, whose aligned
// 8-column scan is cheap and whose 80-register budget is tight; 3 for the 64-bit ones: C4b 4.56 ->
// 4.27 ms, while 3 on the 32-bit path ran 2.80 -> 3.07 ms)
#ifndef R1_NX32
#define R1_NX32 2
#endif
#ifndef R1_NX64
#define R1_NX64 3
#endif
// aligned 4-column groups in the sweep body (128-bit shared loads)
#ifndef R1_V4
#define R1_V4 1
#endif
// two groups (8 columns) per step of the scan loop
#ifndef R1_G8
#define R1_G8 1
#endif
// resident blocks per SM the register budget is sized for (__launch_bounds__ min blocks), per path:
// 3 x 256 threads for the 32-bit tables (85 registers, no spills; 3.47 -> 3.30 ms for C(95,7) on
// B200), 2 for the 64-bit ones (3 spills and runs slower)
// threads per block, per path
#ifndef R1_NT32
#define R1_NT32 256
#endif
#ifndef R1_NT64
#define R1_NT64 256
#endif
#ifndef R1_GBINOM
#define R1_GBINOM 1
#endif
#ifndef R1_MINB32
#define R1_MINB32 3
#endif
#ifndef R1_MINB64
#define R1_MINB64 2
#endif
// 1: count rare-path decisions per block (BlockOut.pad, read by AUTOPIPE_R1_STATS)
#ifndef R1_STATS
#define R1_STATS 0
#endif
struct R1YEntry {      // one y value of the schedule (host-built shard arithmetic, SPEC.md §5)
  int y;               // e_{S-4}
  u32 rows_per_lane;   // R
  u64 row_begin;       // first prefix row (lex rank among P-subsets of {0..y-1}) in the shard
  u64 row_end;         // one past the last
  u64 task_begin;      // global index of this y's first task
  u32 nchunks;         // a row's x range [y+1, L-3] is split into nchunks tasks (long rows only)
  unsigned char xcut[R1_MAXCHUNK + 1];  // chunk c covers x in [xcut[c], xcut[c+1])
  unsigned char pad[7];
};

struct R1Header {
  u64 off;                   // global index of (S, rho = 0, kappa = 0)
  u64 ntasks;
  u64 lo_pre, hi_pre;        // packed prefix cuts of the shard's first / last candidate
  int lo_y, lo_x, lo_e;      // and their (y, x, e)
  int hi_y, hi_x, hi_e;
  int ny;
  u32 counter;               // task counter (reset by the header copy before each launch)
  u32 share;                 // bits: 1 read / 2 publish the grid's best T (theta below); 4 per-task lane seeds always
  u64 theta;                 // smallest T found so far by any lane (UINT64_MAX at launch; atomicMin)
};

template <typename T>
struct __align__(16) ColT {
  T A, K, V, pad;
};
// per-state x table (64-bit): with pcy = PC_{p-1}[y+1] and the lane's row constants
// N0' = min(theta, M_P(1)) + pcy, N1' = min(2 theta, M_P(2)) + pcy, N2' = min(3 theta, M_P(3)) + pcy:
//   stage p-1 fits          <=> pc1 <= N0'   and  lm1 <= theta
//   H1 = min(theta + pcp, N1' + W1),  H2 = min(2 theta + pcp, N2' + W1),  W1 = pcp - pc1 - z1.
struct __align__(16) XT {
  unsigned long long pcp, pc1, lm1;  // PC_p[x+1], PC_{p-1}[x+1], LM_{p-1}[x]
  long long W1;                      // PC_p[x+1] - PC_{p-1}[x+1] - Z_{p-1}[x]
};

typedef long long i64;
// theta >= THETA_ALL means "no best yet": every candidate passes. Real thetas are < 2^59 (the state's
// overflow bound), so theta * 8 and every sum below fit in i64.
constexpr i64 THETA_ALL = 1ll << 60;

__device__ __forceinline__ i64 smin(i64 a, i64 b) { return a < b ? a : b; }

// exact T of an r = 1 candidate (all divisions), from u64 tables (shared memory in the sweep's rare
// path, global memory in the seed kernel: Seed = true gives the seed its own copy, so the sweep's
// call keeps its specialised calling convention)
template <int S, bool Seed = false>
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

// Row terms of one lane, in two parts so that consecutive rows (which usually differ only in the last
// prefix cut) redo two levels, not all of them. Stages 0..P-2 (the "base", cuts e_0..e_{P-2}) give
// M_{P-2}(2..5) and their own feasibility; row_finish adds stage P-1 (cut e_{P-1}) and stage P (cut
// y) and returns whether stages 0..P fit, with N0 = min(theta, M_P(1)), N1 = min(2 theta, M_P(2)),
// N2 = min(3 theta, M_P(3)). P = S-4.
struct RowBase {
  i64 M1, M2, M3, M4, M5;  // M_{P-2}(1..5)
  int a;               // first layer of stage P-1
  bool ok;
};

template <int S>
__device__ __noinline__ void row_base(const u64 *PC, const u64 *Z, const u64 *LM, int L, u64 pre, i64 th,
                                      RowBase &b) {
  constexpr int P = S - 4;
  const int Lp1 = L + 1;
  i64 M[S + 1];
#pragma unroll
  for (int k = 0; k <= S; ++k) M[k] = THETA_ALL * 4;
  bool ok = true;
  int a = 0;
  if (th < THETA_ALL) {
#pragma unroll
    for (int j = 0; j <= P - 2; ++j) {
      const int e = byte_at(pre, j);
      const i64 c = (i64)(PC[j * Lp1 + e + 1] - PC[j * Lp1 + a]);
      const i64 cz = c + (i64)Z[j * L + e];
      ok &= (c <= th) & ((i64)LM[j * L + e] <= th) & (c <= M[1]);
#pragma unroll
      for (int k = 1; k < S - j; ++k) M[k] = smin(th * (1 + k), M[k + 1]) - cz;
      a = e + 1;
    }
  } else {
#pragma unroll
    for (int j = 0; j <= P - 2; ++j) a = byte_at(pre, j) + 1;
  }
  b.M1 = M[1]; b.M2 = M[2]; b.M3 = M[3]; b.M4 = M[4]; b.M5 = M[5];
  b.a = a;
  b.ok = ok;
}

template <int S>
__device__ __forceinline__ bool row_finish(const RowBase &b, const u64 *PC, const u64 *Z, const u64 *LM, int L,
                                           int e1, int y, i64 th, i64 &N0, i64 &N1, i64 &N2) {
  constexpr int P = S - 4;
  if (th >= THETA_ALL) {
    N0 = N1 = N2 = THETA_ALL;
    return true;
  }
  const int Lp1 = L + 1;
  // stage P-1 = [b.a, e1] on worker P-1:  M_{P-1}(k) = min(theta (1+k), M_{P-2}(k+1)) - cz, k = 1..4
  const i64 c1 = (i64)(PC[(P - 1) * Lp1 + e1 + 1] - PC[(P - 1) * Lp1 + b.a]);
  const i64 cz1 = c1 + (i64)Z[(P - 1) * L + e1];
  const i64 M1_1 = smin(2 * th, b.M2) - cz1, M1_2 = smin(3 * th, b.M3) - cz1, M1_3 = smin(4 * th, b.M4) - cz1,
            M1_4 = smin(5 * th, b.M5) - cz1;
  bool ok = b.ok & (c1 <= th) & ((i64)LM[(P - 1) * L + e1] <= th) & (c1 <= b.M1);
  // stage P = [e1+1, y] on worker P
  const i64 c0 = (i64)(PC[P * Lp1 + y + 1] - PC[P * Lp1 + e1 + 1]);
  const i64 cz0 = c0 + (i64)Z[P * L + y];
  ok &= (c0 <= th) & ((i64)LM[P * L + y] <= th) & (c0 <= M1_1);
  N0 = smin(th, smin(2 * th, M1_2) - cz0);
  N1 = smin(2 * th, smin(3 * th, M1_3) - cz0);
  N2 = smin(3 * th, smin(4 * th, M1_4) - cz0);
  return ok;
}

// strict-test threshold for values of type T: "v < thr(h)" == "v <= h"; dead lanes get 0
template <typename T>
__device__ __forceinline__ T thr(i64 h, bool alive) {
  const u64 m = (sizeof(T) == 4) ? 0xFFFFFFFFull : ~0ull;
  if (!alive || h < 0) return (T)0;
  const u64 v = (u64)h + 1;
  return (T)(v > m ? m : v);
}

// A warp's folded column table: A'[e] = (V[e] < THw) ? A[e] : MAX, where THw is the largest strict
// threshold of the warp's lanes. The sweep tests only A'[e] < H1 (one compare per candidate): it is
// a necessary condition of T <= theta (stage p fits and, through the fold, stage q and boundary p
// fit), and every candidate that passes it is re-checked in full (A, K, V) before its exact T.
__device__ __forceinline__ void lds_fold1(unsigned a, u32 &A) { asm("ld.shared.u32 %0, [%1];" : "=r"(A) : "r"(a)); }
__device__ __forceinline__ void lds_fold1(unsigned a, u64 &A) { asm("ld.shared.u64 %0, [%1];" : "=l"(A) : "r"(a)); }
// four consecutive folded columns from a 16-byte-aligned address (32 bytes for 64-bit tables)
__device__ __forceinline__ void lds_group4(unsigned a, u32 (&A)[4]) {
  asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(A[0]), "=r"(A[1]), "=r"(A[2]), "=r"(A[3]) : "r"(a));
}
__device__ __forceinline__ void lds_group4(unsigned a, u64 (&A)[4]) {
  asm("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(A[0]), "=l"(A[1]) : "r"(a));
  asm("ld.shared.v2.u64 {%0, %1}, [%2+16];" : "=l"(A[2]), "=l"(A[3]) : "r"(a));
}
__device__ __forceinline__ u32 warp_max_T(u32 v) { return __reduce_max_sync(0xffffffffu, v); }
__device__ __forceinline__ u64 warp_max_T(u64 v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = umax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// one column of the sweep, read with an explicit 32-bit shared-memory address (one LDS per column
// for 32-bit tables, two for 64-bit ones)
__device__ __forceinline__ void lds_col(unsigned a, u32 &A, u32 &K, u32 &V) {
  u32 pad;
  asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(A), "=r"(K), "=r"(V), "=r"(pad) : "r"(a));
}
__device__ __forceinline__ void lds_col(unsigned a, u64 &A, u64 &K, u64 &V) {
  asm("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(A), "=l"(K) : "r"(a));
  asm("ld.shared.u64 %0, [%1+16];" : "=l"(V) : "r"(a));
}

__device__ __forceinline__ u32 clamp_u32(i64 v) { return v < 0 ? 0u : (v > 0xFFFFFFFFll ? 0xFFFFFFFFu : (u32)v); }

// Per-row constants and the per-x threshold update. Thresholds are for strict tests (v < H <=> v <= h).
template <typename T>
struct XUpd;
template <>
struct XUpd<u64> {  // 64-bit path: thresholds straight from the i64 formulas
  i64 th, N0p, N1p, N2p;
  __device__ __forceinline__ void row(i64 th_, bool alive, i64 N0, i64 N1, i64 N2, u64 pcy) {
    th = th_;
    N0p = alive ? N0 + (i64)pcy : -1;
    N1p = N1 + (i64)pcy;
    N2p = N2 + (i64)pcy;
  }
  __device__ __forceinline__ u64 TH() const { return thr<u64>(th, true); }
  // H1 for the sweep; H2 only on the rare path (the sweep tests A' < H1 alone)
  __device__ __forceinline__ u64 h1(const XT &v) const {
    const bool alive = ((i64)v.pc1 <= N0p) && ((i64)v.lm1 <= th);
    return thr<u64>(smin(th + (i64)v.pcp, N1p + v.W1), alive);
  }
  __device__ __forceinline__ u64 h2(const XT &v) const {
    const bool alive = ((i64)v.pc1 <= N0p) && ((i64)v.lm1 <= th);
    return thr<u64>(smin(2 * th + (i64)v.pcp, N2p + v.W1), alive);
  }
};
template <>
struct XUpd<u32> {  // 32-bit path: every table value is < 2^32 - 16, so clamp once per row and stay in 32 bits
  u32 th1, th2, N0c;
  i64 N1q, N2q;  // N1' + 1, N2' + 1
  __device__ __forceinline__ void row(i64 th, bool alive, i64 N0, i64 N1, i64 N2, u64 pcy) {
    th1 = clamp_u32(th + 1);
    th2 = clamp_u32(2 * th + 1);
    N0c = alive ? clamp_u32(N0 + (i64)pcy + 1) : 0u;
    N1q = N1 + (i64)pcy + 1;
    N2q = N2 + (i64)pcy + 1;
  }
  __device__ __forceinline__ u32 TH() const { return th1; }
  __device__ __forceinline__ u32 h1(const XT &v) const {
    const u32 pcp = (u32)v.pcp;
    const bool alive = ((u32)v.pc1 < N0c) & ((u32)v.lm1 < th1);
    const u32 t1 = min(th1, 0xFFFFFFFFu - pcp) + pcp;  // clamp(theta + 1 + pcp), no overflow
    return alive ? min(t1, clamp_u32(N1q + v.W1)) : 0u;
  }
  __device__ __forceinline__ u32 h2(const XT &v) const {
    const u32 pcp = (u32)v.pcp;
    const bool alive = ((u32)v.pc1 < N0c) & ((u32)v.lm1 < th1);
    const u32 t2 = min(th2, 0xFFFFFFFFu - pcp) + pcp;
    return alive ? min(t2, clamp_u32(N2q + v.W1)) : 0u;
  }
};

template <int S, typename T, int NT>
__global__ void __launch_bounds__(NT, sizeof(T) == 4 ? R1_MINB32 : R1_MINB64) k_search_r1(DevTables g, const R1Header *__restrict__ hdr_g,
                                                     const R1YEntry *__restrict__ yt_g, R1Header *counter_hdr,
                                                     BlockOut *out, int gate) {
  constexpr int p = S - 2, q = S - 1, P = S - 4;
  // gate >= 0: the state was set from device memory and the host launched both paths; only the one
  // the state kernel chose (status bit 1) runs, and neither after an overflow (status bit 0)
  if (gate >= 0 && state_gated_out(g, gate, out)) return;
  extern __shared__ __align__(16) unsigned char smraw[];
  const int L = (int)g.L, Lp1 = L + 1, n = L - 1;
  __shared__ R1Header hdr;
  if (threadIdx.x == 0) hdr = *hdr_g;
  // shared layout: col[n + 16] | xt[n] | PC[S][Lp1] | Z[S-1][L] | LM[S-1][L] | B[Lp1][9] | yt[ny]
  // (col carries 16 sentinel columns past e = L-2 that never pass, so the sweep needs no tail code)
  ColT<T> *col = (ColT<T> *)smraw;
  XT *xt = (XT *)(col + n + 16);
  u64 *PC = (u64 *)(xt + n);
  u64 *Z = PC + S * Lp1;
  u64 *LM = Z + (S - 1) * L;
  u64 *Bn = LM + (S - 1) * L;
  R1YEntry *yt = (R1YEntry *)(Bn + Lp1 * BK8);
  // per-warp folded tables follow the schedule (16-byte aligned)
  const int FN = (n + 16 + 3) & ~3;  // columns per warp table (rows of whole 16-byte units)
  T *foldall = (T *)(((uintptr_t)(yt + hdr_g->ny) + 15) & ~(uintptr_t)15);
#if R1_GBINOM
  for (int i = threadIdx.x; i < Lp1 * BK8; i += NT) Bn[i] = g_binom[i / BK8][i % BK8];
#else
  for (int i = threadIdx.x; i < Lp1 * BK8; i += NT) Bn[i] = c_binom[i / BK8][i % BK8];
#endif
  for (int i = threadIdx.x; i < S * Lp1; i += NT) PC[i] = g.PC[i];
  for (int i = threadIdx.x; i < (S - 1) * L; i += NT) {
    Z[i] = g.Z[i];
    LM[i] = g.LM[i];
  }
  __syncthreads();
  const int ny = hdr.ny;
  for (int i = threadIdx.x; i < ny; i += NT) yt[i] = yt_g[i];
  for (int e = threadIdx.x; e < n + 16; e += NT) {  // per-state column and x tables
    ColT<T> cl;
    if (e < n) {
      const u64 A = PC[p * Lp1 + e + 1];
      const u64 cq = PC[q * Lp1 + L] - PC[q * Lp1 + e + 1];
      cl.A = (T)A;
      cl.K = (T)(A + Z[p * L + e] + cq);
      cl.V = (T)umax(cq, LM[p * L + e]);
      XT xv;
      xv.pcp = A;
      xv.pc1 = PC[(p - 1) * Lp1 + e + 1];
      xv.lm1 = LM[(p - 1) * L + e];
      xv.W1 = (i64)A - (i64)xv.pc1 - (i64)Z[(p - 1) * L + e];
      xt[e] = xv;
    } else {
      cl.A = cl.K = cl.V = (T)~(T)0;  // sentinel: "v < threshold" is false for every threshold
    }
    cl.pad = 0;
    col[e] = cl;
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  T *fold = foldall + (threadIdx.x >> 5) * FN;
  const unsigned fb = (unsigned)__cvta_generic_to_shared(fold);
  T THw_table = (T)0;  // THw the warp's folded table was built for (0 = not built)
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0, nrare = 0;
  const u64 ntasks = hdr.ntasks;
  int yi = 0;
  for (;;) {
    u64 task = 0;
    if (lane == 0) task = atomicAdd(&counter_hdr->counter, 1u);
    task = __shfl_sync(0xffffffffu, task, 0);
    if (task >= ntasks) break;
    // the grid's best T so far (any lane, any block): a candidate with a larger T cannot be the
    // shard's minimum, so every lane may filter against it (non-strict: ties are decided exactly)
    u64 tg = U64MAX;
    if (lane == 0 && (hdr.share & 1)) tg = __ldcg(&counter_hdr->theta);
    tg = __shfl_sync(0xffffffffu, tg, 0);
    const i64 thg = tg < (u64)THETA_ALL ? (i64)tg : THETA_ALL;
    // tasks reach a warp in increasing order, so its cursor only moves forward
    while (yi + 1 < ny && yt[yi + 1].task_begin <= task) ++yi;
    const R1YEntry &ye = yt[yi];
    const int y = ye.y;
    const u64 R = ye.rows_per_lane;
    const u64 local = task - ye.task_begin, grp = local / ye.nchunks;
    const int ch = (int)(local - grp * ye.nchunks);
    const int xa = ye.xcut[ch], xb = ye.xcut[ch + 1];  // this task's x range [xa, xb)
    const u64 r0 = ye.row_begin + grp * 32ull * R + (u64)lane * R;
    const u64 r1 = umin(r0 + R, ye.row_end);
    const u64 pcy = PC[(p - 1) * Lp1 + y + 1];  // start of stage p-1 (warp-uniform)
    u64 pre = (r0 < r1 && P > 0) ? lex_unrank_smem(r0, P, y, Bn) : 0ull;
    // Seed: the lane's first row with the remaining layers split evenly over the last three stages.
    // Its exact T (and index) tightens theta before the sweep, so far fewer candidates reach the rare
    // path while a lane's best is still poor (most visible when a GPU scans a small shard). Only while
    // the grid has no bound (a block too small for the seed kernel), unless share bit 4 forces it.
    if (r0 < r1 && ((hdr.share & 4) || tg == U64MAX)) {
      const int rem = L - 1 - y;  // layers y+1 .. L-1 for stages p-1, p, q
      int xs = y + rem / 3, es = y + (2 * rem) / 3;
      if (xs <= y) xs = y + 1;
      if (es <= xs) es = xs + 1;
      if (es > L - 2) es = L - 2;
      if (xs >= es) xs = es - 1;
      const u64 cuts = pre | ((u64)y << (8 * P)) | ((u64)xs << (8 * (P + 1))) | ((u64)es << (8 * (P + 2)));
      // inside the shard? (only the shard's first and last rows can be partial)
      bool in = true;
      if (pre == hdr.lo_pre && y == hdr.lo_y) in &= (xs > hdr.lo_x) || (xs == hdr.lo_x && es >= hdr.lo_e);
      if (pre == hdr.hi_pre && y == hdr.hi_y) in &= (xs < hdr.hi_x) || (xs == hdr.hi_x && es <= hdr.hi_e);
      if (in) {
        const u64 Ts = exact_T_r1<S>(PC, Z, LM, L, cuts);
        const u64 is = hdr.off + lex_rank_smem(cuts, S - 1, n, Bn);
        if (better(Ts, is, bestT, bestI)) {
          bestT = Ts;
          bestI = is;
        }
      }
    }
    {  // publish the warp's best seed (one atomic per warp, only if it improves the grid's bound)
      u64 wm = bestT;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) wm = umin(wm, __shfl_xor_sync(0xffffffffu, wm, o));
      if (lane == 0 && wm < tg && (hdr.share & 2)) atomicMin(&counter_hdr->theta, wm);
    }
    // strictness: theta = best while this lane's task may still hold a smaller index than its best
    bool strict = true;
    if (r0 < r1 && bestT != U64MAX) {
      // a lower bound of the lane's first candidate in this task (non-strict is always safe)
      const u64 first = pre | ((u64)y << (8 * P)) | ((u64)xa << (8 * (P + 1))) | ((u64)(xa + 1) << (8 * (P + 2)));
      strict = hdr.off + lex_rank_smem(first, S - 1, n, Bn) > bestI;
    }
    // evaluated candidates of this task: the (x, e) pairs y < x < e <= L-2 of the x chunk in each of
    // the lane's rows, restricted on the shard's first / last row (at most one of each per shard:
    // the lo row is row_begin of y = lo_y, the hi row is row_end - 1 of y = hi_y)
    const bool task_lo = r0 < r1 && y == hdr.lo_y && r0 == ye.row_begin;
    const bool task_hi = r0 < r1 && y == hdr.hi_y && r1 == ye.row_end;
    if (r0 < r1) {
      // rank of the pair (x, e) among the row's pairs (closed form)
      auto prank = [&](int x, int e) -> u64 {
        const u64 a = (u64)(x - y - 1), m1 = (u64)(L - 3 - y);  // m1 = pairs with x = y + 1
        return a * m1 - a * (a - 1) / 2 + (u64)(e - x - 1);
      };
      const u64 flo = prank(xa, xa + 1), fhi = prank(xb, xb + 1);  // this task's x chunk
      const u64 lo1 = task_lo ? umax(flo, prank(hdr.lo_x, hdr.lo_e)) : flo;
      const u64 hi1 = task_hi ? umin(fhi, prank(hdr.hi_x, hdr.hi_e) + 1) : fhi;
      const u64 full = fhi - flo, nrows = r1 - r0;
      if (nrows == 1) {
        cnt += hi1 > lo1 ? hi1 - lo1 : 0ull;
      } else {
        cnt += (nrows - 2) * full + (fhi > lo1 ? fhi - lo1 : 0ull) + (hi1 > flo ? hi1 - flo : 0ull);
      }
    }
    RowBase base;
    bool need_base = true;
    for (u64 row = r0;; ++row) {
      const bool active = row < r1;
      if (!__any_sync(0xffffffffu, active)) break;
      // partial rows at the shard boundaries: (x, e) range restricted, checked on the rare path
      const bool lo_part = task_lo && row == r0, hi_part = task_hi && row + 1 == r1;
      i64 th = (bestT == U64MAX) ? THETA_ALL : (i64)bestT - (strict ? 1 : 0);
      if (thg < th) th = thg;
      bool aliveP = false;
      i64 N0 = 0, N1 = 0, N2 = 0;
      if (active) {
        if (need_base) row_base<S>(PC, Z, LM, L, pre, th, base);
        aliveP = row_finish<S>(base, PC, Z, LM, L, byte_at(pre, P - 1), y, th, N0, N1, N2);
      }
      XUpd<T> xu;
      xu.row(th, aliveP && active, N0, N1, N2, pcy);
      T TH = active ? xu.TH() : (T)0;
      {  // (re)build the warp's folded table when the warp's largest threshold changed
        const T THw = warp_max_T(TH);
        if (THw != THw_table) {
          for (int e = lane; e < FN; e += 32) {
            const ColT<T> c = col[e < n + 16 ? e : n + 15];
            fold[e] = (c.V < THw) ? c.A : (T)~(T)0;
          }
          __syncwarp();
          THw_table = THw;
        }
      }
      // ---- x sweep (warp-uniform), then the hot column sweep -------------------------------
      constexpr unsigned FS = sizeof(T);
      const int cend = L - 1;  // columns e <= L-2
      // Rare path: candidate (xk, ee) passed the sweep's filter; check it in full and decide it
      // exactly. Afterwards every later candidate of this lane in index order is larger, so theta
      // becomes strict (best - 1) and the row terms are recomputed (the caller refreshes thresholds).
      auto rare = [&](int xk, int ee, const T h1) -> bool {
        const ColT<T> c = col[ee];
        if (!((c.A < h1) & (c.V < TH))) return false;
        if (!(c.K < xu.h2(xt[xk]))) return false;
        if (lo_part && (xk < hdr.lo_x || (xk == hdr.lo_x && ee < hdr.lo_e))) return false;
        if (hi_part && (xk > hdr.hi_x || (xk == hdr.hi_x && ee > hdr.hi_e))) return false;
        const u64 cuts = pre | ((u64)y << (8 * P)) | ((u64)xk << (8 * (P + 1))) | ((u64)ee << (8 * (P + 2)));
        const u64 Tc = exact_T_r1<S>(PC, Z, LM, L, cuts);
        const u64 idx = hdr.off + lex_rank_smem(cuts, S - 1, n, Bn);
#if R1_STATS
        ++nrare;
#endif
        if (better(Tc, idx, bestT, bestI)) {
          bestT = Tc;
          bestI = idx;
        }
        strict = true;
        th = (i64)bestT - 1;
        if (thg < th) th = thg;
        row_base<S>(PC, Z, LM, L, pre, th, base);
        aliveP = row_finish<S>(base, PC, Z, LM, L, byte_at(pre, P - 1), y, th, N0, N1, N2);
        xu.row(th, aliveP, N0, N1, N2, pcy);
        TH = xu.TH();
        return true;
      };
      const unsigned aend = fb + (unsigned)cend * FS;
      // one x from column c0 to the end (the deferred x of a pass), four columns per step;
      // the threshold is refreshed after every decision
      auto sweep1 = [&](int xk, int c0) {
        const XT xv = xt[xk];
        T H1 = xu.h1(xv);
        for (unsigned a = fb + (unsigned)c0 * FS; a < aend; a += 4 * FS) {
          T A4[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) lds_fold1(a + u * FS, A4[u]);
          const bool hit = (A4[0] < H1) | (A4[1] < H1) | (A4[2] < H1) | (A4[3] < H1);
          if (hit) {
            const int c = (int)((a - fb) / FS);
            for (int u = 0; u < 4; ++u)
              if (A4[u] < H1 && rare(xk, c + u, H1)) H1 = xu.h1(xv);
          }
        }
      };
      // NX x values per pass: x .. x+NX-1 test the same columns, so one broadcast load serves NX
      // candidates and their compare chains are independent. Hits of the first x are decided at
      // once; a later x only records its first hit and is rescanned (sweep1) after the pass, in x
      // order, so a lane decides its candidates in increasing index order (tie-break, reading C-13).
      constexpr int NX = sizeof(T) == 4 ? R1_NX32 : R1_NX64;
      for (int x = xa; x < xb; x += NX) {
        const int nx = xb - x < NX ? xb - x : NX;
        T H1[NX];
        int first[NX];
#pragma unroll
        for (int k = 0; k < NX; ++k) {
          H1[k] = (k < nx) ? xu.h1(xt[x + k]) : (T)0;
          first[k] = cend;
        }
        auto refresh = [&]() {
#pragma unroll
          for (int k = 0; k < NX; ++k)
            if (k < nx) H1[k] = xu.h1(xt[x + k]);
        };
        // head: columns x+1 .. x+NX-1 (column e belongs to the x+k with e > x+k)
#pragma unroll
        for (int j = 1; j < NX; ++j) {
          const int c = x + j;
          if (c < cend) {
            T A0;
            lds_fold1(fb + (unsigned)c * FS, A0);
            if (A0 < H1[0] && rare(x, c, H1[0])) refresh();
#pragma unroll
            for (int k = 1; k < j; ++k)
              if (first[k] == cend && A0 < H1[k]) first[k] = c;
          }
        }
        // 64-bit tables: every column from x+NX on belongs to every x of the pass (4 columns per step,
        // four 64-bit loads; the sentinel columns past L-2 never pass)
        auto body64 = [&]() {
          for (unsigned a = fb + (unsigned)(x + NX) * FS; a < aend; a += 4 * FS) {
            T A4[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) lds_fold1(a + u * FS, A4[u]);
            bool h[NX];
#pragma unroll
            for (int k = 0; k < NX; ++k) h[k] = (A4[0] < H1[k]) | (A4[1] < H1[k]) | (A4[2] < H1[k]) | (A4[3] < H1[k]);
            bool any = h[0];
#pragma unroll
            for (int k = 1; k < NX; ++k) any |= h[k];
            if (any) {
              const int c = (int)((a - fb) / FS);
              if (h[0])
                for (int u = 0; u < 4; ++u)
                  if (A4[u] < H1[0] && rare(x, c + u, H1[0])) refresh();
#pragma unroll
              for (int k = 1; k < NX; ++k)
                if (h[k] && first[k] == cend) first[k] = c;
            }
          }
        };
#if R1_V4
        // body: every column from cs = x+NX on belongs to every x of the pass. Columns go in aligned
        // groups of 4 (one 128-bit shared load on the 32-bit path); the first group starts at cs
        // rounded down, its columns below cs masked to MAX; the sentinel columns past L-2 never pass.
        // The scan loop only tests the group's minimum against Hm, the largest threshold still
        // live (H1[0], and H1[k] of a later x until its first hit is recorded): one compare per group
        // and no branch into the hit code until something passes.
        const int cs = x + NX;
        if constexpr (sizeof(T) != 4) {
          body64();
        } else if (cs < cend) {
          T Hm;
          auto set_hm = [&]() {
            Hm = H1[0];
#pragma unroll
            for (int k = 1; k < NX; ++k)
              if (first[k] == cend && H1[k] > Hm) Hm = H1[k];
          };
          set_hm();
          auto group = [&](unsigned o, const T (&A4)[4]) {
            const int c = (int)(o / FS);
            if ((A4[0] < H1[0]) | (A4[1] < H1[0]) | (A4[2] < H1[0]) | (A4[3] < H1[0]))
              for (int u = 0; u < 4; ++u)
                if (A4[u] < H1[0] && rare(x, c + u, H1[0])) refresh();
#pragma unroll
            for (int k = 1; k < NX; ++k)
              if (first[k] == cend && ((A4[0] < H1[k]) | (A4[1] < H1[k]) | (A4[2] < H1[k]) | (A4[3] < H1[k])))
                first[k] = c > cs ? c : cs;
            set_hm();
          };
          const unsigned oend = (unsigned)cend * FS;
          unsigned o = (unsigned)(cs & ~3) * FS;
          T A4[4];
          lds_group4(fb + o, A4);
          {
            const int d = cs & 3;
            if (d > 0) A4[0] = (T)~(T)0;
            if (d > 1) A4[1] = (T)~(T)0;
            if (d > 2) A4[2] = (T)~(T)0;
          }
          for (;;) {
            if (min(min(A4[0], A4[1]), min(A4[2], A4[3])) < Hm) group(o, A4);
            o += 4 * FS;
            if (o >= oend) break;
            // tight scan to the next group with a column below Hm
#if R1_G8
            // (two groups per step: one compare per 8 columns; the sentinels cover the overrun)
            T B4[4];
            bool hitb = false;
            for (;;) {
              lds_group4(fb + o, A4);
              lds_group4(fb + o + 4 * FS, B4);
              if (min(min(min(A4[0], A4[1]), min(A4[2], A4[3])), min(min(B4[0], B4[1]), min(B4[2], B4[3]))) < Hm) {
                hitb = true;
                break;
              }
              o += 8 * FS;
              if (o >= oend) break;
            }
            if (!hitb) break;
            if (min(min(A4[0], A4[1]), min(A4[2], A4[3])) < Hm) group(o, A4);
            o += 4 * FS;
            if (o >= oend) break;
#pragma unroll
            for (int u = 0; u < 4; ++u) A4[u] = B4[u];
#else
            for (;;) {
              lds_group4(fb + o, A4);
              if (min(min(A4[0], A4[1]), min(A4[2], A4[3])) < Hm) break;
              o += 4 * FS;
              if (o >= oend) break;
            }
            if (o >= oend) break;
#endif
          }
        }
#else
        body64();
#endif
#pragma unroll
        for (int k = 1; k < NX; ++k)
          if (first[k] < cend) sweep1(x + k, first[k]);
      }
      // ---- next row of this lane: lexicographic successor of the prefix below y ------------
      // usually only the last prefix cut moves (+1): the base (stages 0..P-2) stays valid
      need_base = false;
      if (active && row + 1 < r1) {
        if (byte_at(pre, P - 1) < y - 1) {
          pre += 1ull << (8 * (P - 1));
        } else {
          lex_next_packed(pre, P, y);
          need_base = true;
        }
      }
    }
    {  // publish the warp's best after the task (one reduction-atomic per warp and task: a
       // per-improvement atomic on one address serialises at L2 and costs more than it saves)
      u64 wm = bestT;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) wm = umin(wm, __shfl_xor_sync(0xffffffffu, wm, o));
      if (lane == 0 && wm < tg && (hdr.share & 2)) atomicMin(&counter_hdr->theta, wm);
    }
  }
  block_minloc_store<NT>(bestT, bestI, cnt, out + blockIdx.x);
  // diagnostics: rare-path decisions of the block (BlockOut.pad; read by AUTOPIPE_R1_STATS)
  nrare = warp_sum(nrare);
  __shared__ u64 rs[NT / 32];
  if ((threadIdx.x & 31) == 0) rs[threadIdx.x >> 5] = nrare;
  __syncthreads();
  if (threadIdx.x == 0) {
    u64 t = 0;
    for (int i = 0; i < NT / 32; ++i) t += rs[i];
    out[blockIdx.x].pad = t;
  }
}

// ------------------------------------------------------------------------------------------------
// Seed bound (before the sweep; same stream): a good in-shard candidate found by a cheap heuristic
// gives the grid's shared theta a tight start, so the sweep's early rows are not flooded with rare-path
// decisions while the lanes' own bests are still poor. It never changes a result: theta is the T of a
// real candidate of the shard, the sweep still decides every candidate against the running theta
// (non-strict against the shared value), and the shard's (T, index) minimum has T <= theta.
// One warp per variant: the first cut free (v = 0) or fixed next to the shard's first / last cut
// (v = 1..4). The rest of the cuts: the min-max greedy (each stage as long as its cost c_s and its
// boundary term lm_s stay <= theta), theta found by a 33-way parallel search over the warp; then up to
// R1_SEED_ROUNDS rounds of the best single-cut move (+-1, +-2) by exact T, moves kept inside the shard.
// ------------------------------------------------------------------------------------------------
#ifndef R1_SEED_ROUNDS
#define R1_SEED_ROUNDS 4
#endif

template <int S>
__device__ __forceinline__ bool cuts_in_shard(const R1Header &h, const int *c) {
  constexpr int P = S - 4;
  int lo[S - 1], hi[S - 1];
#pragma unroll
  for (int i = 0; i < P; ++i) {
    lo[i] = (int)((h.lo_pre >> (8 * i)) & 0xFF);
    hi[i] = (int)((h.hi_pre >> (8 * i)) & 0xFF);
  }
  lo[P] = h.lo_y; lo[P + 1] = h.lo_x; lo[P + 2] = h.lo_e;
  hi[P] = h.hi_y; hi[P + 1] = h.hi_x; hi[P + 2] = h.hi_e;
  int cl = 0, ch = 0;  // lexicographic comparison against lo and hi (first differing cut decides)
#pragma unroll
  for (int i = 0; i < S - 1; ++i) {
    if (cl == 0 && c[i] != lo[i]) cl = c[i] < lo[i] ? -1 : 1;
    if (ch == 0 && c[i] != hi[i]) ch = c[i] < hi[i] ? -1 : 1;
  }
  return cl >= 0 && ch <= 0;
}

// greedy cuts for stages j..S-1 (stage s on worker s) over layers [a, L-1] under theta; false if some
// stage cannot be placed. Cut s is the largest e with c_s <= theta, backed off while lm_s(e) > theta,
// leaving one layer per later stage.
template <int S>
__device__ bool greedy_cuts(const DevTables &g, int L, int j, int a, u64 th, int *c) {
  const int Lp1 = L + 1;
  int pos = a;
  for (int s = j; s < S - 1; ++s) {
    const u64 *pc = g.PC + (size_t)s * Lp1;
    const int emax = L - 1 - (S - 1 - s);
    if (pos > emax) return false;
    const u64 lim = pc[pos] + th;
    int lo = pos - 1, hi = emax;  // largest e in [pos, emax] with pc[e + 1] <= lim (binary search)
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (pc[mid + 1] <= lim) lo = mid;
      else hi = mid - 1;
    }
    int e = lo;
    while (e >= pos && g.LM[(size_t)s * L + e] > th) --e;
    if (e < pos) return false;
    c[s] = e;
    pos = e + 1;
  }
  return g.PC[(size_t)(S - 1) * Lp1 + L] - g.PC[(size_t)(S - 1) * Lp1 + pos] <= th;
}

template <int S>
__device__ __forceinline__ u64 pack_cuts(const int *c) {
  u64 p = 0;
#pragma unroll
  for (int i = 0; i < S - 1; ++i) p |= (u64)c[i] << (8 * i);
  return p;
}

template <int S>
__global__ void __launch_bounds__(160) k_seed_r1(DevTables gd, R1Header *hdr) {
  if (gd.status[0] & 1) return;  // overflowing state: the search kernels exit too
  // the walks below are chains of dependent loads: stage PC (stages 0..S-1), Z and LM in shared memory
  __shared__ u64 sPC[S * (MAXL + 1)], sZ[(S - 1) * MAXL], sLM[(S - 1) * MAXL];
  const int L = (int)gd.L, Lp1 = L + 1, lane = threadIdx.x & 31, v = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < S * Lp1; i += blockDim.x) sPC[i] = gd.PC[i];
  for (int i = threadIdx.x; i < (S - 1) * L; i += blockDim.x) {
    sZ[i] = gd.Z[i];
    sLM[i] = gd.LM[i];
  }
  __syncthreads();
  DevTables g = gd;
  g.PC = sPC;
  g.Z = sZ;
  g.LM = sLM;
  const R1Header h = *hdr;
  const int lo0 = (int)(h.lo_pre & 0xFF), hi0 = (int)(h.hi_pre & 0xFF);
  int j = 0, e0 = 0;
  if (v > 0) {
    j = 1;
    e0 = v == 1 ? lo0 : v == 2 ? lo0 + 1 : v == 3 ? hi0 - 1 : hi0;
    if (e0 < 0 || e0 > L - S || (v == 2 && e0 > hi0) || (v == 3 && e0 < lo0)) return;
  }
  const int a = j ? e0 + 1 : 0;
  // theta range: [0, an upper bound that is feasible]
  u64 tlo = 0, thi = 0;
  for (int s = 0; s < S; ++s) thi = umax(thi, g.PC[(size_t)s * Lp1 + L]);
  for (int s = 0; s < S - 1; ++s)
    for (int e = lane; e < L; e += 32) thi = umax(thi, g.LM[(size_t)s * L + e]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) thi = umax(thi, __shfl_xor_sync(0xffffffffu, thi, o));
  int c[S - 1];
  if (j) c[0] = e0;
  if (!greedy_cuts<S>(g, L, j, a, thi, c)) return;
  while (thi - tlo > 1) {  // invariant: tlo infeasible (or 0), thi feasible
    const u64 step = (thi - tlo) / 33 ? (thi - tlo) / 33 : 1;
    const u64 t = tlo + step * (u64)(lane + 1);
    int cc[S - 1];
    if (j) cc[0] = e0;
    const bool ok = t < thi && greedy_cuts<S>(g, L, j, a, t, cc);
    const unsigned m = __ballot_sync(0xffffffffu, ok);
    const unsigned bad = __ballot_sync(0xffffffffu, !ok && t < thi);
    if (m) {
      const int f = __ffs(m) - 1;  // the smallest feasible t
      thi = __shfl_sync(0xffffffffu, t, f);
      const unsigned below = bad & ((1u << f) - 1u);
      if (below) tlo = __shfl_sync(0xffffffffu, t, 31 - __clz(below));
    } else {
      const unsigned lastbad = bad ? 31 - __clz(bad) : 0;
      tlo = bad ? __shfl_sync(0xffffffffu, t, lastbad) : tlo;
      if (!bad) break;
    }
  }
  if (j) c[0] = e0;
  greedy_cuts<S>(g, L, j, a, thi, c);
  u64 bestT = cuts_in_shard<S>(h, c) ? exact_T_r1<S, true>(g.PC, g.Z, g.LM, L, pack_cuts<S>(c)) : U64MAX;
  // refinement: lane m tries move m (cut i = j + m / 4, delta -2, -1, +1, +2); the best improving
  // in-shard move of the warp is applied
  for (int round = 0; round < R1_SEED_ROUNDS; ++round) {
    int cc[S - 1];
#pragma unroll
    for (int i = 0; i < S - 1; ++i) cc[i] = c[i];
    const int i = j + lane / 4, d = (lane & 3) < 2 ? (lane & 3) - 2 : (lane & 3) - 1;
    u64 T = U64MAX;
    if (i < S - 1) {
      cc[i] += d;
      const int lo = i == 0 ? 0 : cc[i - 1] + 1, hi = i == S - 2 ? L - 2 : cc[i + 1] - 1;
      if (cc[i] >= lo && cc[i] <= hi && cuts_in_shard<S>(h, cc)) T = exact_T_r1<S, true>(g.PC, g.Z, g.LM, L, pack_cuts<S>(cc));
    }
    u64 bt = T;
    int bl = lane;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const u64 t2 = __shfl_xor_sync(0xffffffffu, bt, o);
      const int l2 = __shfl_xor_sync(0xffffffffu, bl, o);
      if (t2 < bt || (t2 == bt && l2 < bl)) { bt = t2; bl = l2; }
    }
    if (bt >= bestT) break;
    bestT = bt;
    const int bi = j + bl / 4, bd = (bl & 3) < 2 ? (bl & 3) - 2 : (bl & 3) - 1;
    c[bi] += bd;
  }
  if (lane == 0 && bestT != U64MAX) atomicMin(&hdr->theta, (unsigned long long)bestT);
}

// ------------------------------------------------------------------------------------------------
// host side: the task schedule (rows per y restricted to the shard) and the launch
// ------------------------------------------------------------------------------------------------
static u64 env_u64(const char *name, u64 dflt) {  // tuning knobs (AUTOPIPE_EXPERIMENTS=1 only)
  const char *v = experiment_knob(name);
  return (v && *v) ? strtoull(v, nullptr, 10) : dflt;
}

// host binomials C(n, k), n < 256, k <= 8 (exact in u64), built once
static u64 g_hb[256][9];
static void init_hb() {
  static bool done = false;
  if (done) return;
  for (int n = 0; n < 256; ++n)
    for (int k = 0; k < 9; ++k) g_hb[n][k] = (k == 0) ? 1 : (n == 0 ? 0 : g_hb[n - 1][k - 1] + g_hb[n - 1][k]);
  done = true;
}
static inline u64 hb(int n, int k) { return (k < 0 || n < 0 || k > n) ? 0 : g_hb[n][k]; }

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

// Cross-shard bound (row e): k_theta_out folds a shard's seed T into a caller's device word (atomicMin;
// the caller min-reduces it over ranks), k_theta_in lowers a sweep's shared theta to such a word
// before the sweep starts. theta is always the exact T of a real candidate of some shard.
__global__ void k_theta_out(const R1Header *hdr, u64 *theta) {
  if (threadIdx.x == 0) atomicMin((unsigned long long *)theta, (unsigned long long)hdr->theta);
}
__global__ void k_theta_in(R1Header *hdr, const u64 *bound) {
  if (threadIdx.x == 0) {
    const u64 b = *bound;
    if (b < hdr->theta) hdr->theta = b;
  }
}

// prep = false: the schedule for this (S, shard) was just built and copied by the launch of the other
// path (gate >= 0 launches both); reuse it
template <int S, typename T>
static int launch_r1_t(const DevTables &g, const SearchSpace &sp, u64 k_begin, u64 k_end, int sms,
                       BlockOut *out, int max_blocks, int *nblocks, void *work, void *pinned, size_t work_bytes,
                       cudaStream_t st, int gate, bool prep, const R1Ext &ext) {
  constexpr int P = S - 4, NT = sizeof(T) == 4 ? R1_NT32 : R1_NT64;
  const int L = (int)g.L, n = L - 1, k = S - 1;
  unsigned char *hbuf = (unsigned char *)pinned + (size_t)S * 16384;
  R1Header *h = (R1Header *)hbuf;
  int ny = 0;
  u64 tasks = 0;
  if (prep) {
    init_hb();
    int lo[8], hi[8];
    host_unrank(k_begin, k, n, lo);
    host_unrank(k_end - 1, k, n, hi);
    R1YEntry *yt = (R1YEntry *)(hbuf + sizeof(R1Header));
    memset(h, 0, sizeof(*h));
    h->theta = env_u64("AUTOPIPE_R1_THETA0", U64MAX);  // experiment knob: a known bound (unset: none)
    // per-task lane seeds (bit 4) only while the grid has no bound yet: once the seed kernel has set
    // theta they cost more than they tighten (B200: C(95,7) 2.81 -> 2.73 ms, 8-way shard 0.64 -> 0.58)
    static const u64 share = env_u64("AUTOPIPE_R1_SHARE", 3);
    h->share = (u32)share;
    h->off = sp.off[S];
    for (int i = 0; i < P; ++i) {
      h->lo_pre |= (u64)lo[i] << (8 * i);
      h->hi_pre |= (u64)hi[i] << (8 * i);
    }
    h->lo_y = lo[P]; h->lo_x = lo[P + 1]; h->lo_e = lo[P + 2];
    h->hi_y = hi[P]; h->hi_x = hi[P + 1]; h->hi_e = hi[P + 2];
    // Task size by estimated cost (thread-instructions per lane): a row costs ~150 (prefix terms) +
    // ~26 per x + ~6 per candidate. The target per lane-task is set so the shard splits into ~40 tasks
    // per resident warp (2 x 8 warps per SM): the dynamic schedule's tail stays small at any shard size
    // (a full 96-layer space on one GPU, or 1/8 of it per GPU), and the per-task unrank is amortised.
    u64 rb_[256], re_[256], cost_[256];
    u64 total_cost = 0;
    for (int y = P; y <= L - 4; ++y) {
      // rows (prefix, y) whose candidates intersect [lo, hi]: a contiguous range of prefix ranks
      const bool lo_fits = (P == 0) || lo[P - 1] < y;
      const bool hi_fits = (P == 0) || hi[P - 1] < y;
      rb_[y] = count_less(y, P, lo) + ((lo_fits && y < lo[P]) ? 1 : 0);
      re_[y] = count_less(y, P, hi) + ((hi_fits && y <= hi[P]) ? 1 : 0);
      const u64 m = (u64)(L - 2 - y);
      cost_[y] = 150 + 26 * (m - 1) + 6 * (m * (m - 1) / 2);
      if (re_[y] > rb_[y]) total_cost += (re_[y] - rb_[y]) * cost_[y];
    }
    static const u64 tpw = env_u64("AUTOPIPE_R1_TPW", 30), min_target = env_u64("AUTOPIPE_R1_MINTARGET", 12000);
    const u64 lane_tasks = (u64)sms * 16 * 32 * tpw;
    u64 TARGET = total_cost / (lane_tasks ? lane_tasks : 1);
    // Floor on the task size: 12,000 amortises the per-task unrank and seed, but a small space (a
    // 21-26-layer model) would then be a handful of tasks on 2-6 blocks, latency-bound for 100-300 us.
    // Small spaces get tasks sized to give every resident warp slot about two (floor 300).
    u64 floor_t = min_target;
    const u64 fill = total_cost / ((u64)sms * 16 * 32 * 2);
    if (fill < floor_t) floor_t = fill > 300 ? fill : 300;
    if (TARGET < floor_t) TARGET = floor_t;
    // Guided sizes: warps take tasks in schedule order, so the kernel ends about one task length after
    // the last task starts. Tasks in the final 15 % of the cost shrink linearly to 1/4 of the target
    // (smaller ones pay more per-task overhead than they save in tail; measured on B200).
    static const u64 guided = env_u64("AUTOPIPE_R1_GUIDED", 2);
    u64 cum = 0;
    for (int y = P; y <= L - 4; ++y) {
      const u64 rb = rb_[y], re = re_[y];
      if (re <= rb) continue;
      const u64 row_cost = cost_[y];
      u64 tgt = TARGET;
      if (guided && total_cost) {
        const double frac = (double)cum / (double)total_cost, left = 1.0 - frac;
        const double zone = guided == 1 ? 0.25 : 0.15, floor_ = guided == 1 ? 1.0 / 16 : 0.25;
        if (left < zone) {
          const double g = left / zone > floor_ ? left / zone : floor_;
          tgt = (u64)((double)TARGET * g);
          if (tgt < 1) tgt = 1;
        }
      }
      cum += (re - rb) * row_cost;
      const u64 R = row_cost >= tgt ? 1 : (tgt + row_cost - 1) / row_cost;
      R1YEntry &ye = yt[ny++];
      memset(&ye, 0, sizeof(ye));
      // a row longer than the target is split into x chunks of about equal candidate counts, so a
      // small shard still gives every warp many tasks (a whole row can hold ~4000 candidates)
      const int x_first = y + 1, x_end = L - 2;  // x in [y+1, L-3]
      static const u64 max_chunks = env_u64("AUTOPIPE_R1_CHUNKS", 16);
      u64 nch = row_cost > tgt ? (row_cost + tgt - 1) / tgt : 1;
      if (nch > max_chunks) nch = max_chunks;
      if (nch > (u64)R1_MAXCHUNK) nch = R1_MAXCHUNK;
      if (nch > (u64)(x_end - x_first)) nch = (u64)(x_end - x_first);
      if (nch < 1) nch = 1;
      const u64 m = (u64)(L - 2 - y), pairs = m * (m - 1) / 2;
      int nc = 0;
      ye.xcut[nc++] = (unsigned char)x_first;
      u64 acc = 0;
      for (int x = x_first; x < x_end && nc < (int)nch; ++x) {
        acc += (u64)(L - 2 - x);  // pairs with this x
        if (acc * nch >= pairs * (u64)nc && x + 1 < x_end) ye.xcut[nc++] = (unsigned char)(x + 1);
      }
      ye.xcut[nc] = (unsigned char)x_end;
      const u64 nt = (re - rb + 32 * R - 1) / (32 * R);
      ye.y = y;
      ye.rows_per_lane = (u32)R;
      ye.row_begin = rb;
      ye.row_end = re;
      ye.task_begin = tasks;
      ye.nchunks = (u32)nc;
      tasks += nt * (u64)nc;
    }
    h->ny = ny;
    h->ntasks = tasks;
  } else {
    ny = h->ny;
    tasks = h->ntasks;
  }
  *nblocks = 0;
  if (tasks == 0) return 0;
  const size_t hbytes = sizeof(R1Header) + (size_t)ny * sizeof(R1YEntry);
  // one 16 KB slot per S, so the launches of one search never share a schedule buffer
  if ((size_t)(S + 1) * 16384 > work_bytes || hbytes > 16384) return 0;
  work = (unsigned char *)work + (size_t)S * 16384;
  // the schedule is staged in the context's pinned buffer (one 16 KB slot per S, like the device work
  // area), so the copy is a true async DMA and never waits for earlier work on the stream
  int launched = 1;  // the sweep kernel below, + the seed kernel
  if (ext.theta_out) {  // seed only (autopipe_search_seed_async): the seed's T into the caller's word
    cudaMemcpyAsync(work, hbuf, hbytes, cudaMemcpyHostToDevice, st);
    if (k_end - k_begin < (1ull << 26)) return 0;
    k_seed_r1<S><<<1, 160, 0, st>>>(g, (R1Header *)work);
    k_theta_out<<<1, 32, 0, st>>>((const R1Header *)work, ext.theta_out);
    return 2;
  }
  if (prep && ext.bound) {  // a bound from every shard's seed replaces this shard's own seed
    cudaMemcpyAsync(work, hbuf, hbytes, cudaMemcpyHostToDevice, st);
    k_theta_in<<<1, 32, 0, st>>>((R1Header *)work, ext.bound);
    ++launched;
  } else if (prep) {
    cudaMemcpyAsync(work, hbuf, hbytes, cudaMemcpyHostToDevice, st);
    // before the sweep, on its stream. (Beside it, on a stream of its own with a block slot left free,
    // it came too late for the 32-bit C4a search: 3.08 ms against 2.85.) Experiment knob: 0 = off.
    static const u64 seed = env_u64("AUTOPIPE_R1_SEED", 1);
    // a small block (a short model's space, C2/C3) is over before a bad start costs anything, while
    // the seed's ~20 us would sit on its critical path
    if (seed && k_end - k_begin >= (1ull << 26)) {
      k_seed_r1<S><<<1, 160, 0, st>>>(g, (R1Header *)work);
      ++launched;
    }
  }
  const size_t smem = (size_t)(n + 16) * sizeof(ColT<T>) + (size_t)n * sizeof(XT) + (size_t)S * (L + 1) * 8 +
                      2 * (size_t)(S - 1) * L * 8 + (size_t)(L + 1) * BK8 * 8 + (size_t)ny * sizeof(R1YEntry) + 16 +
                      (size_t)(NT / 32) * (size_t)((n + 16 + 3) & ~3) * sizeof(T);
  // the attribute and the occupancy query cost microseconds each: redo them only when smem changes
  // (per device: a process may drive several GPUs, one context each)
  static size_t smem_set[64] = {0};
  static int per_sm_dev[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  if (smem != smem_set[dev]) {
    cudaFuncSetAttribute(k_search_r1<S, T, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int q = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&q, k_search_r1<S, T, NT>, NT, smem);
    per_sm_dev[dev] = q < 1 ? 1 : q;
    smem_set[dev] = smem;
  }
  const int per_sm = per_sm_dev[dev];
  u64 blocks = (u64)sms * per_sm;
  const u64 need = (tasks + (NT / 32) - 1) / (NT / 32);
  if (blocks > need) blocks = need;
  if (blocks > (u64)max_blocks) blocks = (u64)max_blocks;
  const R1Header *hd = (const R1Header *)work;
  const R1YEntry *yd = (const R1YEntry *)((unsigned char *)work + sizeof(R1Header));
  k_search_r1<S, T, NT><<<(unsigned)blocks, NT, smem, st>>>(g, hd, yd, (R1Header *)work, out, gate);
  *nblocks = (int)blocks;
  return launched;
}

template <typename T>
static int launch_r1_s(int S, const DevTables &g, const SearchSpace &sp, u64 a, u64 b, int sms, BlockOut *out,
                       int mb, int *nb, void *w, void *pin, size_t wb, cudaStream_t st, int gate, bool prep,
                       const R1Ext &x) {
  switch (S) {
    case 5: return launch_r1_t<5, T>(g, sp, a, b, sms, out, mb, nb, w, pin, wb, st, gate, prep, x);
    case 6: return launch_r1_t<6, T>(g, sp, a, b, sms, out, mb, nb, w, pin, wb, st, gate, prep, x);
    case 7: return launch_r1_t<7, T>(g, sp, a, b, sms, out, mb, nb, w, pin, wb, st, gate, prep, x);
    case 8: return launch_r1_t<8, T>(g, sp, a, b, sms, out, mb, nb, w, pin, wb, st, gate, prep, x);
  }
  *nb = 0;
  return 0;
}

int launch_search_r1(const DevTables &g, const SearchSpace &sp, int S, u64 k_begin, u64 k_end, int path32,
                     int sms, BlockOut *out, int max_blocks, int *nblocks, void *work, void *pinned,
                     size_t work_bytes, cudaStream_t st, const R1Ext &ext) {
  if (ext.theta_out) {  // seed only: no sweep, the 64-bit tables serve either path
    *nblocks = 0;
    return launch_r1_s<u64>(S, g, sp, k_begin, k_end, sms, out, max_blocks, nblocks, work, pinned, work_bytes, st,
                            -1, true, ext);
  }
  if (path32 == 1)
    return launch_r1_s<u32>(S, g, sp, k_begin, k_end, sms, out, max_blocks, nblocks, work, pinned, work_bytes, st,
                            -1, true, ext);
  if (path32 == 0)
    return launch_r1_s<u64>(S, g, sp, k_begin, k_end, sms, out, max_blocks, nblocks, work, pinned, work_bytes, st,
                            -1, true, ext);
  // path unknown on the host (state set from device memory, asynchronous search): both paths, each
  // gated on the state kernel's choice; one schedule serves both
  int n32 = 0, n64 = 0;
  int k = launch_r1_s<u32>(S, g, sp, k_begin, k_end, sms, out, max_blocks, &n32, work, pinned, work_bytes, st, 1, true,
                           ext);
  if (n32 > 0)
    k += launch_r1_s<u64>(S, g, sp, k_begin, k_end, sms, out + n32, max_blocks - n32, &n64, work, pinned, work_bytes,
                          st, 0, false, ext);
  *nblocks = n32 + n64;
  return k;
}

void upload_binomials_r1(const u64 (*tab)[BINOM_K]) { upload_binomials_tu(tab); }

}  // namespace ap
