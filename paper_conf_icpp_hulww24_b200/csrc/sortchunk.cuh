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

// Shape of a record: S and the number of extra replicas (sum r - S), 64 buckets. Records of one
// shape run the same stage, replica and boundary loops, so a warp of them does not diverge.
__device__ __forceinline__ u32 shape_key(const uint4 &r) {
  const u32 S = r.x & 0xFFu;
  const u32 n = (u32)(__popc(__vcmpne4(r.z, 0xFFFFFFFFu)) + __popc(__vcmpne4(r.w, 0xFFFFFFFFu))) >> 3;
  return ((S & 7u) << 3) | ((n - S) & 7u);
}

// f(record, global index) for every record of recs[0, count), block-strided over chunks; every thread
// of the block must call it (it synchronises the block).
template <typename F>
__device__ __forceinline__ void for_each_sorted(const uint4 *__restrict__ recs, u64 count, F &&f) {
  __shared__ uint4 srec[EV_CH];
  __shared__ u32 sidx[EV_CH];
  __shared__ u32 hist[EV_NB];
  const int tid = threadIdx.x;
  const u64 nch = (count + EV_CH - 1) / EV_CH;
  for (u64 ch = blockIdx.x; ch < nch; ch += gridDim.x) {
    const u64 base = ch * EV_CH;
    if (tid < EV_NB) hist[tid] = 0;
    __syncthreads();
    uint4 rr[EV_PER];
    u32 key[EV_PER], rank[EV_PER];
#pragma unroll
    for (int j = 0; j < EV_PER; ++j) {
      const u64 i = base + (u64)(j * 256 + tid);
      key[j] = EV_NB;
      rank[j] = 0;
      if (i < count) {
        rr[j] = __ldg(recs + i);
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
