// k_eval.cu — batched scoring of explicit partition records (autopipe_eval_partitions) and RL
// rollout rewards (autopipe_rollout_rewards). Rows a4-a8 for explicit records.
//
// Launch: a persistent grid (a multiple of the SM count) of 256-thread blocks, grid-stride over
// records. Each block stages the state tables into shared memory once (PF, PB, PP, O, G, tau), then
// every thread scores one record per iteration: one 128-bit load of the 16-byte record
// (ld.global.nc), the closed form of SPEC.md §4 in registers, one 8-byte store per output. Loads and
// stores of consecutive threads are consecutive: 512 B of records in and 256 B of times out per warp.
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
// MODE: the schedule of the model (row f3; SCHED_PIPEDREAM is the 1F1B closed form of rows a4-a7).
template <bool ROLLOUT, bool P32, int MODE>
__global__ void __launch_bounds__(256, MODE == SCHED_PIPEDREAM ? EVAL_MINB : 2) k_eval(DevTables g, const uint4 *__restrict__ recs, u64 count,
                                              u64 *__restrict__ out_t, u64 *__restrict__ out_sw,
                                              CurPart cur, ModelP m) {
  extern __shared__ u64 sm[];
  const SmemTab t = stage_tables(g, sm);
  const int L = t.L, N = (int)g.N;
  // a state that failed the device-side overflow check (set_state_device) scores nothing
  const bool overflow = (g.status[0] & 1ull) != 0;
  const u64 stride = (u64)gridDim.x * blockDim.x;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
    const uint4 r = __ldg(recs + i);
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
}

static int grid_for(u64 count, int sms) {
  const u64 need = (count + 255) / 256;
  const u64 cap = (u64)sms * 8;  // up to 8 resident 256-thread blocks per SM
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
