// common.cuh — device-side data layout and integer helpers of the AutoPipe cost-model engine.
//
// Everything is unsigned integer arithmetic (SPEC.md: times in ns, bytes, inverse bandwidth in
// fs/byte). The host (autopipe.cu) guarantees, through the overflow checks of set_state, that every
// sum formed here is < 2^59 and every bytes*tau product is < 2^64, so u64 is exact throughout.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ap {

typedef unsigned long long u64;
typedef unsigned int u32;

constexpr int MAXS = 8;       // stages of a 16-byte record (C-15)
constexpr int MAXN = 8;       // workers of a 16-byte record
constexpr int MAXSW = 16;     // stages of a 32-byte wide record (row f4)
constexpr int MAXNW = 16;     // workers of a state and of a wide record (row f4)
constexpr int TAUW = 16;      // row stride of the padded tau table
constexpr int MAXL = 255;     // layers
constexpr int BINOM_N = 256;  // C(n, k) for n < 256
constexpr int BINOM_K = 17;   // k <= 16 (wide spaces, row f4; saturated at UINT64_MAX)
constexpr int BK8 = 9;        // columns k <= 8 staged in shared memory for 16-byte spaces
constexpr u64 U64MAX = ~0ull;

// Global-memory tables written by the state kernels (k_state.cu) and read by every scoring kernel.
// All arrays are row-major; "Lp1" = L + 1 (exclusive prefix sums have L + 1 entries).
struct DevTables {
  u32 L, N, Lp1, pad;
  u64 *PF;    // [N][L+1]  exclusive prefix of fp_ns per worker          (row a1)
  u64 *PB;    // [N][L+1]  exclusive prefix of bp_ns per worker          (row a1)
  u64 *PC;    // [N][L+1]  exclusive prefix of fp_ns + bp_ns (r = 1 stage cost)
  u64 *PP;    // [L+1]     exclusive prefix of weight bytes              (row a1)
  u64 *O;     // [L]       activation bytes
  u64 *G;     // [L]       input-gradient bytes
  u64 *tau;   // [16][16]  fs per byte, row u -> column v (padded to 16 x 16)
  u64 *Z;     // [7][L]    r = 1 boundary s (worker s -> s+1) cut after layer l: cf + cb   (row a2)
  u64 *LM;    // [7][L]    ... max(cf, cb)                                                (row a2)
  u32 *PC32;  // [N][L+1]  32-bit copies for the 32-bit search path (valid iff path32)
  u64 *ring;  // [256]     slowest link of the ring over each worker set (N <= 8; ascending ring order)
  u64 *xp;    // [L-1][16][16][2] single-worker boundary at cut l, sender u, receiver v:
              //   {xfer(O[l], tau[u][v]), xfer(G[l+1], tau[v][u])} (forward, backward)
  u32 *PF32;  // [N][L+1]  32-bit copies of PF, PB for the narrow eval path (valid iff status bit 2)
  u32 *PB32;
  u32 *Z32;   // [7][L]
  u32 *LM32;  // [7][L]
  u64 *status; // [2] written by the state kernel: [0] bit0 = overflow, bit1 = 32-bit path,
               // bit2 = narrow (per-worker stage sums < 2^31 - 16, O and G < 2^31, tau < 2^32); [1] = bound
};

// The model a scoring call evaluates (NEXT row f3, reading F-3; autopipe_set_schedule).
enum { SCHED_PIPEDREAM = 0, SCHED_2BW = 1, SCHED_GPIPE = 2, SCHED_DAPPLE = 3, SCHED_RR = 4, SCHED_CHIMERA = 5 };
enum { SYNC_RING = 0, SYNC_PS = 1 };
struct ModelP {
  u32 sched;      // SCHED_*
  u32 sync;       // SYNC_*: how a replicated stage synchronises its gradients
  u32 M;          // micro-batches per iteration (1 for PipeDream)
  u32 recompute;  // GPipe: the backward op re-runs the forward
};

__host__ __device__ __forceinline__ u64 umax(u64 a, u64 b) { return a > b ? a : b; }
__host__ __device__ __forceinline__ u64 umin(u64 a, u64 b) { return a < b ? a : b; }

// ceil(x / 10^6) for the transfer time xfer(x, tau) = ceil(x * tau / 1e6) (SPEC.md §1, C-7).
__device__ __forceinline__ u64 xfer_fs(u64 p) { return (p + 999999ull) / 1000000ull; }
__device__ __forceinline__ u64 xfer(u64 bytes, u64 fs_per_byte) {
  return xfer_fs(bytes * fs_per_byte);  // the product is < 2^64 (set_state check)
}

// floor(x / d) for a runtime divisor d in [1, MAXD] (a replica count; MAXD = 8 for the 16-byte
// records, 16 for the wide ones) and x < 2^63, by Granlund-Montgomery with N = 63:
// m = ceil(2^(63+l) / d), l = ceil(log2 d), q = mulhi(x, m) >> (l - 1); exact for every x < 2^63
// (d = 1 is the identity). The multiplier is chosen once per divisor, hoisted out of the loops over
// replicas and shards.
struct __align__(16) DivEnt {  // DivR's multipliers for one divisor (see DivR and Div32)
  u64 m;
  u32 sh, Ms;
  u32 m32, k32, pad0, pad1;
};
constexpr int DIVTAB_WORDS = 4 * (MAXNW + 1);  // u64 words of the table for d = 0..16 (entry 0 unused)

template <int MAXD = 8>
struct DivR {
  u64 m;
  u32 sh, d, Ms;
  __device__ __forceinline__ explicit DivR(u32 d_) : d(d_) {
    if (MAXD <= 8) {
      m = (d == 3u || d == 6u) ? 0xaaaaaaaaaaaaaaabull
        : (d == 5u)            ? 0xcccccccccccccccdull
        : (d == 7u)            ? 0x924924924924924aull
                               : 0x8000000000000000ull;
      sh = (d <= 2u) ? 0u : (d <= 4u) ? 1u : 2u;
    } else {
      m = (d == 3u || d == 6u || d == 12u) ? 0xaaaaaaaaaaaaaaabull
        : (d == 5u || d == 10u)            ? 0xcccccccccccccccdull
        : (d == 7u || d == 14u)            ? 0x924924924924924aull
        : (d == 9u)                        ? 0xe38e38e38e38e38full
        : (d == 11u)                       ? 0xba2e8ba2e8ba2e8cull
        : (d == 13u)                       ? 0x9d89d89d89d89d8aull
        : (d == 15u)                       ? 0x8888888888888889ull
                                           : 0x8000000000000000ull;
      sh = (d <= 2u) ? 0u : (d <= 4u) ? 1u : (d <= 8u) ? 2u : 3u;
    }
    // floor(k / d) for 0 <= k < 256: (k * ceil(2^16 / d)) >> 16 is exact on that range
    Ms = (d == 1u) ? 65536u : (d == 2u) ? 32768u : (d == 3u) ? 21846u : (d == 4u) ? 16384u
       : (d == 5u) ? 13108u : (d == 6u) ? 10923u : (d == 7u) ? 9363u : 8192u;
    if (MAXD > 8 && d > 8u)
      Ms = (d == 9u) ? 7282u : (d == 10u) ? 6554u : (d == 11u) ? 5958u : (d == 12u) ? 5462u
         : (d == 13u) ? 5042u : (d == 14u) ? 4682u : (d == 15u) ? 4370u : 4096u;
  }
  // the same multipliers from a table of the 16 divisors staged in shared memory (stage_tables):
  // one 16-byte shared load instead of the select chains above
  __device__ __forceinline__ DivR(u32 d_, const DivEnt *tab) : d(d_) {
    const DivEnt e = tab[d_];
    m = e.m;
    sh = e.sh;
    Ms = e.Ms;
  }
  __device__ __forceinline__ u64 div(u64 x) const { return d == 1u ? x : (__umul64hi(x, m) >> sh); }
  __device__ __forceinline__ u64 ceil(u64 x) const { return div(x + d - 1); }
  __device__ __forceinline__ u32 small(u32 k) const { return (k * Ms) >> 16; }
};
typedef DivR<8> Div8;

// floor(x / d) for d in [1, 16] and 32-bit x < 2^31 (the narrow path: a state whose per-worker
// stage sums stay below 2^31): m = ceil(2^(31 + c) / d) < 2^32 with c = ceil(log2 d),
// q = mulhi32(x, m) >> (c - 1). Exact for every x < 2^31 (the error m d - 2^(31+c) < d <= 2^c);
// tools/check_div32.py checks it exhaustively on the top of the range.
struct Div32 {
  u32 m, k, d;
  __host__ __device__ __forceinline__ static void make(u32 d_, u32 &m_, u32 &k_) {
    if (d_ <= 1u) { m_ = 0u; k_ = 0u; return; }
    u32 c = 0;
    while ((1u << c) < d_) ++c;
    m_ = (u32)((((unsigned long long)1 << (31 + c)) + d_ - 1) / d_);
    k_ = c - 1;
  }
  __device__ __forceinline__ Div32(u32 d_, const DivEnt *tab) : d(d_) {
    m = tab[d_].m32;
    k = tab[d_].k32;
  }
  __device__ __forceinline__ u32 div(u32 x) const { return d == 1u ? x : (__umulhi(x, m) >> k); }
  __device__ __forceinline__ u32 ceil(u32 x) const { return div(x + d - 1); }
};


__device__ __forceinline__ int byte_at(u64 v, int i) { return (int)((v >> (8 * i)) & 0xFF); }

// Lexicographic (time, index) minimum used by every argmin (reading C-13: smallest index wins ties).
struct MinLoc {
  u64 t, idx;
};
__device__ __forceinline__ bool better(u64 t1, u64 i1, u64 t2, u64 i2) {
  return t1 < t2 || (t1 == t2 && i1 < i2);
}
__device__ __forceinline__ void warp_minloc(u64 &t, u64 &idx) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const u64 t2 = __shfl_xor_sync(0xffffffffu, t, o);
    const u64 i2 = __shfl_xor_sync(0xffffffffu, idx, o);
    if (better(t2, i2, t, idx)) { t = t2; idx = i2; }
  }
}
__device__ __forceinline__ u64 warp_sum(u64 v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Block-level (time, index) minimum + evaluated count; thread 0 writes the block's entry.
// Deterministic: the lexicographic min and the integer sum do not depend on the order.
struct BlockOut {
  u64 t, idx, count, pad;
};
// Device-side path choice for a search launched before the host knows the state's path (state set
// from device memory, asynchronous search): the launcher enqueues the kernel of each path with
// gate = 1 (32-bit) or 0 (64-bit); a block whose path the state kernel did not choose, or any block
// after an overflowing state, writes an empty result and returns (uniformly, before any barrier).
__device__ __forceinline__ bool state_gated_out(const DevTables &g, int gate, BlockOut *out) {
  const u64 s = *(volatile const u64 *)g.status;
  if (!(s & 1) && (int)((s >> 1) & 1) == gate) return false;
  if (threadIdx.x == 0) {
    out[blockIdx.x].t = U64MAX;
    out[blockIdx.x].idx = U64MAX;
    out[blockIdx.x].count = 0;
    out[blockIdx.x].pad = 0;
  }
  return true;
}

template <int NT>
__device__ __forceinline__ void block_minloc_store(u64 t, u64 idx, u64 cnt, BlockOut *dst) {
  __shared__ u64 st[NT / 32], si[NT / 32], sc[NT / 32];
  warp_minloc(t, idx);
  cnt = warp_sum(cnt);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) { st[wid] = t; si[wid] = idx; sc[wid] = cnt; }
  __syncthreads();
  if (wid == 0) {
    t = (lane < NT / 32) ? st[lane] : U64MAX;
    idx = (lane < NT / 32) ? si[lane] : U64MAX;
    cnt = (lane < NT / 32) ? sc[lane] : 0;
    warp_minloc(t, idx);
    cnt = warp_sum(cnt);
    if (lane == 0) { dst->t = t; dst->idx = idx; dst->count = cnt; }
  }
}

}  // namespace ap
