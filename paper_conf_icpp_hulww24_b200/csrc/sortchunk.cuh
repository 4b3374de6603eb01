// sortchunk.cuh — shape-ordered traversal of a batch of partition records (k_eval).
//
// Random rollout records mix S = 1..8 and replica counts; scored in input order, a warp runs the
// union of its lanes' stage, replica and boundary loops (ncu: ~9 of 32 lanes active). A warp here
// takes chunks of consecutive records (coalesced 128-bit loads), counts them into shape buckets in
// its slice of shared memory, and hands them to the scoring function in bucket order, so the lanes
// of a step score records of (nearly) one shape. Every record is still scored exactly once, and its
// outputs go to its own position (8-byte stores scattered within the chunk).
#pragma once
#include <type_traits>

#include "common.cuh"

namespace ap {

constexpr int EV_NB = 64;              // shape buckets
// equal record ranges per warp for 16-byte records (B200: S = 8 r = 1 GPT-96 records 90 -> 74 us per
// 1M, C5 -1 %); chunks from a global counter for the wide ones, whose costs vary more (static was 10 %
// slower there)
template <typename Rec>
struct EvalStatic {
  static constexpr bool value = sizeof(Rec) == 16;
};
#ifndef EVAL_PER16
#define EVAL_PER16 8                   // 16-byte records per lane and warp chunk (B200 C5: 8 beat 4 by 5 %)
#endif

struct Rec16 {  // a 16-byte partition record
  uint4 a;
};
struct Rec32 {  // a 32-byte wide partition record (row f4)
  uint4 a, b;
};
__device__ __forceinline__ Rec16 load_rec(const Rec16 *p) { return Rec16{__ldg(&p->a)}; }
__device__ __forceinline__ Rec32 load_rec(const Rec32 *p) { return Rec32{__ldg(&p->a), __ldg(&p->b)}; }

__device__ __forceinline__ u32 workers_named(u32 v) { return (u32)__popc(__vcmpne4(v, 0xFFFFFFFFu)) >> 3; }

// Shape of a record: S and the number of extra replicas (sum r - S), 64 buckets. Records of one
// shape run the same stage, replica and boundary loops, so a warp of them does not diverge.
__device__ __forceinline__ u32 shape_key(const Rec16 &r) {
  const u32 S = r.a.x & 0xFFu;
  const u32 n = workers_named(r.a.z) + workers_named(r.a.w);
  return ((S & 7u) << 3) | ((n - S) & 7u);
}
// wide records: S in 1..16 (4 bits) and extra replicas 0, 1, 2, >= 3 (2 bits)
__device__ __forceinline__ u32 shape_key(const Rec32 &r) {
  const u32 S = r.a.x & 0xFFu;
  const u32 n = workers_named(r.b.x) + workers_named(r.b.y) + workers_named(r.b.z) + workers_named(r.b.w);
  const u32 extra = n - S;  // wraps for an invalid record: any bucket is fine
  return (((S - 1u) & 15u) << 2) | (extra < 3u ? extra : 3u);
}

// f(record, global index) for every record of recs[0, count). Each warp works on its own: it takes
// a chunk of 32 * PER consecutive records from a global counter (dynamic schedule: no tail of idle
// warps whatever the batch size), loads it with coalesced 128-bit loads, counting-sorts it by shape
// in its own slice of shared memory (no block barrier: a warp that drew cheap records moves on to the
// next chunk at once) and scores it in shape order, 32 records per step. *counter must be 0 at
// launch; NW = warps per block.
template <int NW, typename Rec>
struct WarpSort {
  static constexpr int PER = sizeof(Rec) == 16 ? EVAL_PER16 : 4;  // records per lane and chunk
  static constexpr int CH = 32 * PER;
};

// f(Rec &slot, u64 i) scores the record in `slot` (global index i) and may overwrite the slot with its
// results; store(const Rec &slot, u64 i), when given, then writes every slot of the chunk in input
// order — consecutive lanes, consecutive records: coalesced stores (row a8).
struct NoStore {
  template <typename Rec>
  __device__ void operator()(const Rec &, u64) const {}
};
// DYNAMIC forces the chunk counter for 16-byte records too (scoring costs that vary by orders of
// magnitude between records: round-robin replicas).
template <int NW, typename Rec, bool DYNAMIC = false, typename F, typename G = NoStore>
__device__ __forceinline__ void for_each_sorted_warp(const Rec *__restrict__ recs, u64 count, u32 *counter, F &&f,
                                                     G store = G()) {
  constexpr int PER = WarpSort<NW, Rec>::PER, CH = WarpSort<NW, Rec>::CH;
  __shared__ Rec srec[NW][CH];
  __shared__ unsigned short sidx[NW][CH];
  __shared__ u32 hist[NW][EV_NB];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const u64 nch = (count + CH - 1) / CH;
  Rec *sr = srec[w];
  unsigned short *si = sidx[w];
  u32 *h = hist[w];
  // static split: warp gw of W takes records [count gw / W, count (gw + 1) / W), in chunks of CH
  // (the same number of records per warp); dynamic: chunks of CH from the global counter
  constexpr bool STATIC = EvalStatic<Rec>::value && !DYNAMIC;
  const u64 W = (u64)gridDim.x * NW, gw = (u64)blockIdx.x * NW + w;
  const u64 r1 = STATIC ? count * (gw + 1) / W : count;
  u64 base = STATIC ? count * gw / W : 0;
  for (;; base += CH) {
    if (STATIC) {
      if (base >= r1) break;
    } else {
      u32 c = 0;
      if (lane == 0) c = atomicAdd(counter, 1u);
      c = __shfl_sync(0xffffffffu, c, 0);
      if ((u64)c >= nch) break;
      base = (u64)c * CH;
    }
    const u64 cend = (r1 - base < (u64)CH) ? r1 : base + CH;
    h[lane] = 0;
    h[lane + 32] = 0;
    __syncwarp();
    // records go to shared memory in input order right away (no register copy); a lane keeps only
    // key | rank << 8 per record, and the sort writes the permutation sorted slot -> input slot
    u32 kr[PER];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const u64 i = base + (u64)(j * 32 + lane);
      kr[j] = EV_NB;
      if (i < cend) {
        const Rec r = load_rec(recs + i);
        sr[j * 32 + lane] = r;
        const u32 key = shape_key(r);
        kr[j] = key | (atomicAdd(&h[key], 1u) << 8);
      }
    }
    __syncwarp();
    {  // exclusive scan of the 64 bucket counts, two per lane
      const u32 a = h[2 * lane], b2 = h[2 * lane + 1];
      u32 v = a + b2;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const u32 y = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += y;
      }
      const u32 ex = v - (a + b2);
      __syncwarp();
      h[2 * lane] = ex;
      h[2 * lane + 1] = ex + a;
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      const u32 key = kr[j] & 0xFFu;
      if (key < EV_NB) si[h[key] + (kr[j] >> 8)] = (unsigned short)(j * 32 + lane);
    }
    __syncwarp();
    const u32 nvalid = (u32)(cend - base);
#pragma unroll 1
    for (int j = 0; j < PER; ++j) {
      const u32 slot = (u32)(j * 32 + lane);
      if (slot < nvalid) {
        const u32 src = si[slot];
        f(sr[src], base + src);
      }
    }
    if constexpr (!std::is_same<G, NoStore>::value) {
      __syncwarp();
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        const u32 q = (u32)(j * 32 + lane);
        if (q < nvalid) store(sr[q], base + q);
      }
    }
    __syncwarp();  // the next chunk reuses this warp's slice
  }
}

}  // namespace ap
