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
#include "sortchunk.cuh"

namespace ap {

struct CurPart {
  u64 cuts, masks;
  int S, valid;
};

#ifndef EVAL_MINB
#define EVAL_MINB 4
#endif
// 1: each block scores its records in chunks sorted by shape (sortchunk.cuh)
#ifndef EVAL_SORT
#define EVAL_SORT 1
#endif
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
  for_each_sorted(recs, count, [&](const uint4 &r, u64 i) {
    score_one<ROLLOUT, P32, MODE>(t, L, N, overflow, r, i, out_t, out_sw, cur, m);
  });
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
