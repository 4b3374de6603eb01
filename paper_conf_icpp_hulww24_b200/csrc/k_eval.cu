// k_eval.cu — batched scoring of explicit partition records (autopipe_eval_partitions) and RL
// rollout rewards (autopipe_rollout_rewards). Rows a4-a8 for explicit records.
//
// Launch: a persistent grid (one wave of resident 256-thread blocks) striding over chunks of 1024
// records. Each block stages the state tables into shared memory once (PF, PB, PP, O, G, tau), loads
// a chunk with coalesced 128-bit loads (ld.global.nc), sorts it by shape in shared memory (a
// counting sort over 64 buckets), and every thread scores records of one shape: the closed form of
// SPEC.md §4 in registers, one 8-byte store per output at the record's position.
// Invalid records (SPEC.md §2) score UINT64_MAX and never fail the batch.
#include "eval.cuh"
#include "internal.h"
#include "sched.cuh"

namespace ap {

struct CurPart {
  u64 cuts, masks;
  int S, valid;
};

#ifndef EVAL_MINB
#define EVAL_MINB 4
#endif
// 1: each block scores its records in chunks sorted by shape (see k_eval)
#ifndef EVAL_SORT
#define EVAL_SORT 1
#endif
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

template <bool ROLLOUT, bool P32, int MODE>
__device__ __forceinline__ void score_one(const SmemTab &t, int L, int N, bool overflow, const uint4 &r, u64 i,
                                          u64 *__restrict__ out_t, u64 *__restrict__ out_sw, const CurPart &cur,
                                          const ModelP &m) {
  const u64 lo = (u64)r.x | ((u64)r.y << 32), hi = (u64)r.z | ((u64)r.w << 32);
  int S;
  u64 cuts, masks;
  u64 T = U64MAX, sw = U64MAX;
  if (!overflow && decode_record(lo, hi, L, N, S, cuts, masks)) {
    T = model_time<MODE, P32>(t, S, cuts, masks, m);
    if (ROLLOUT) sw = switch_bytes(t, S, cuts, masks, cur.S, cur.cuts, cur.masks);
  }
  out_t[i] = T;
  if (ROLLOUT) out_sw[i] = sw;
}

// MODE: the schedule of the model (row f3; SCHED_PIPEDREAM is the 1F1B closed form of rows a4-a7).
// With EVAL_SORT a block takes chunks of EV_CH consecutive records (coalesced 128-bit loads), counts
// them into shape buckets in shared memory, and scores them in bucket order: random rollout records
// mix S = 1..8 and replica counts, and scoring them in input order left ~9 of 32 lanes active
// (ncu); in bucket order the warps run uniform loop trip counts. Each time goes back to the
// record's own position (8-byte scattered stores within the chunk).
template <bool ROLLOUT, bool P32, int MODE>
__global__ void __launch_bounds__(256, MODE == SCHED_PIPEDREAM ? EVAL_MINB : 2)
    k_eval(DevTables g, const uint4 *__restrict__ recs, u64 count, u64 *__restrict__ out_t, u64 *__restrict__ out_sw,
           CurPart cur, ModelP m) {
  extern __shared__ u64 sm[];
  const SmemTab t = stage_tables(g, sm);
  const int L = t.L, N = (int)g.N;
  // a state that failed the device-side overflow check (set_state_device) scores nothing
  const bool overflow = (g.status[0] & 1ull) != 0;
#if EVAL_SORT
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
      if (slot < nvalid)
        score_one<ROLLOUT, P32, MODE>(t, L, N, overflow, srec[slot], base + sidx[slot], out_t, out_sw, cur, m);
    }
    __syncthreads();  // the next chunk reuses srec / sidx / hist
  }
#else
  const u64 stride = (u64)gridDim.x * blockDim.x;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
    score_one<ROLLOUT, P32, MODE>(t, L, N, overflow, __ldg(recs + i), i, out_t, out_sw, cur, m);
#endif
}

static int grid_for(u64 count, int sms) {
  const u64 per = EVAL_SORT ? (u64)EV_CH : 256;  // records per block and step
  const u64 need = (count + per - 1) / per;
  const u64 cap = (u64)sms * (EVAL_SORT ? EVAL_MINB : 8);  // one wave of resident blocks
  return (int)(need < cap ? (need ? need : 1) : cap);
}

template <bool ROLLOUT, bool P32, int MODE>
static void run_eval(int grid, size_t smem, cudaStream_t st, const DevTables &g, const void *recs, u64 count,
                     u64 *out_t, u64 *out_sw, const CurPart &cur, const ModelP &m) {
  k_eval<ROLLOUT, P32, MODE><<<grid, 256, smem, st>>>(g, (const uint4 *)recs, count, out_t, out_sw, cur, m);
}

template <bool ROLLOUT>
static void dispatch_eval(int grid, size_t smem, cudaStream_t st, const DevTables &g, const void *recs, u64 count,
                          u64 *out_t, u64 *out_sw, const CurPart &cur, const ModelP &m, int path32) {
  switch (m.sched) {
    case SCHED_2BW: run_eval<ROLLOUT, false, SCHED_2BW>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m); break;
    case SCHED_GPIPE: run_eval<ROLLOUT, false, SCHED_GPIPE>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m); break;
    case SCHED_DAPPLE: run_eval<ROLLOUT, false, SCHED_DAPPLE>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m); break;
    default:
      if (path32) run_eval<ROLLOUT, true, SCHED_PIPEDREAM>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m);
      else run_eval<ROLLOUT, false, SCHED_PIPEDREAM>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m);
  }
}

int launch_eval(const DevTables &g, const void *recs, u64 count, u64 *out_t, u64 *out_sw,
                const int *cur_S, const u64 *cur_cuts, const u64 *cur_masks, int path32, const ModelP &m, int sms,
                cudaStream_t st) {
  if (count == 0) return 0;
  const size_t smem = (size_t)smem_words(g.L, g.N) * sizeof(u64);
  CurPart cur{0, 0, 0, 0};
  if (cur_S) {
    cur.S = *cur_S;
    cur.cuts = *cur_cuts;
    cur.masks = *cur_masks;
    cur.valid = 1;
  }
  const int grid = grid_for(count, sms);
  if (out_sw) dispatch_eval<true>(grid, smem, st, g, recs, count, out_t, out_sw, cur, m, path32);
  else dispatch_eval<false>(grid, smem, st, g, recs, count, out_t, nullptr, cur, m, path32);
  return 1;
}

}  // namespace ap
