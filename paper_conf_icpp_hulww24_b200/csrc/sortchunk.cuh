// sortchunk.cuh — shape-ordered traversal of a batch of partition records (k_eval, k_switch).
//
// Random rollout records mix S = 1..8 and replica counts; scored in input order, a warp runs the
// union of its lanes' stage, replica and boundary loops (ncu: ~9 of 32 lanes active). A block here
// takes chunks of EV_CH consecutive records (coalesced 128-bit loads), counts them into shape buckets
// in shared memory, and hands them to the scoring function in bucket order, so a warp scores records
// of one shape. Every record is still scored exactly once, and its outputs go to its own position
// (8-byte stores scattered within the chunk).
#pragma once
#include "common.cuh"

namespace ap {

constexpr int EV_PER = 4;              // records per thread and chunk
constexpr int EV_CH = 256 * EV_PER;    // records per chunk
constexpr int EV_NB = 64;              // shape buckets

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

// f(record, global index) for every record of recs[0, count), block-strided over chunks; every thread
// of the block must call it (it synchronises the block).
template <typename Rec, typename F>
__device__ __forceinline__ void for_each_sorted(const Rec *__restrict__ recs, u64 count, F &&f) {
  __shared__ Rec srec[EV_CH];
  __shared__ u32 sidx[EV_CH];
  __shared__ u32 hist[EV_NB];
  const int tid = threadIdx.x;
  const u64 nch = (count + EV_CH - 1) / EV_CH;
  for (u64 ch = blockIdx.x; ch < nch; ch += gridDim.x) {
    const u64 base = ch * EV_CH;
    if (tid < EV_NB) hist[tid] = 0;
    __syncthreads();
    Rec rr[EV_PER];
    u32 key[EV_PER], rank[EV_PER];
#pragma unroll
    for (int j = 0; j < EV_PER; ++j) {
      const u64 i = base + (u64)(j * 256 + tid);
      key[j] = EV_NB;
      rank[j] = 0;
      if (i < count) {
        rr[j] = load_rec(recs + i);
        key[j] = shape_key(rr[j]);
        rank[j] = atomicAdd(&hist[key[j]], 1u);
      }
    }
    __syncthreads();
    if (tid < 32) {  // exclusive scan of the 64 bucket counts, two per lane
      const u32 a = hist[2 * tid], b = hist[2 * tid + 1];
      u32 v = a + b;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const u32 y = __shfl_up_sync(0xffffffffu, v, o);
        if (tid >= o) v += y;
      }
      const u32 ex = v - (a + b);
      hist[2 * tid] = ex;
      hist[2 * tid + 1] = ex + a;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < EV_PER; ++j) {
      if (key[j] < EV_NB) {
        const u32 slot = hist[key[j]] + rank[j];
        srec[slot] = rr[j];
        sidx[slot] = (u32)(j * 256 + tid);
      }
    }
    __syncthreads();
    const u64 left = count - base;
    const u32 nvalid = left < (u64)EV_CH ? (u32)left : (u32)EV_CH;
#pragma unroll 1
    for (int j = 0; j < EV_PER; ++j) {
      const u32 slot = (u32)(j * 256 + tid);
      if (slot < nvalid) f(srec[slot], base + sidx[slot]);
    }
    __syncthreads();  // the next chunk reuses srec / sidx / hist
  }
}

}  // namespace ap
