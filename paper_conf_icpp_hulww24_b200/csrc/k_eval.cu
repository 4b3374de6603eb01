// k_eval.cu — batched scoring of explicit partition records (autopipe_eval_partitions) and RL
// rollout rewards (autopipe_rollout_rewards). Rows a4-a8 for explicit records.
//
// Launch: a persistent grid (one wave of resident 256-thread blocks). Each block stages the state
// tables into shared memory once (PF, PB, PP, O, G, tau, the divisor table); then every warp on its
// own takes an equal share of the records in chunks of 256 (128 wide ones), loads them with coalesced
// 128-bit loads (ld.global.nc), counting-sorts them by shape in its slice of shared memory
// (sortchunk.cuh) and scores them 32 at a time in shape order: the closed form of SPEC.md §4 in
// registers, the results written back into the records' shared-memory slots and stored in input
// order (consecutive lanes, consecutive 8-byte outputs: coalesced).
// Invalid records (SPEC.md §2) score UINT64_MAX and never fail the batch.
#include <cstring>

#include "eval.cuh"
#include "internal.h"
#include "sched.cuh"
#include "sortchunk.cuh"

namespace ap {

struct CurPart {  // the current partition of a rollout (16-byte or wide)
  P8 p8;
  P16 p16;
  int S, valid;
};

// resident blocks per SM for the wide (P16) GPipe / DAPPLE evals, whose 16-stage max-plus state
// spills at the 2-block register budget
#ifndef EVAL_MINB_WF
#define EVAL_MINB_WF 2
#endif
// resident blocks per SM for the round-robin evals (a latency-bound recurrence in local memory)
#ifndef EVAL_MINB_CH
#define EVAL_MINB_CH 2  // B200, 1M Chimera records: 1 / 2 / 3 blocks per SM within 0.5 % (4.44 / 4.44 / 4.42 ms)
#endif
#ifndef EVAL_MINB_RR
#define EVAL_MINB_RR 2
#endif
#define EVAL_BLOCKS(MODE, P)                                                                    \
  ((MODE == SCHED_PIPEDREAM && P::MS == 8) ? EVAL_MINB                                          \
   : (P::MS == 16 && (MODE == SCHED_GPIPE || MODE == SCHED_DAPPLE)) ? EVAL_MINB_WF              \
   : (MODE == SCHED_RR) ? EVAL_MINB_RR : (MODE == SCHED_CHIMERA) ? EVAL_MINB_CH : 2)
#ifndef EVAL_MINB
#define EVAL_MINB 4
#endif
constexpr int EVAL_NT = 256;
// Decode + validate + score one record; Rec16 -> P8 (16-byte records), Rec32 -> P16 (wide, row f4).
__device__ __forceinline__ bool decode_any(const Rec16 &r, int L, int N, int &S, P8 &p) {
  return decode_record((u64)r.a.x | ((u64)r.a.y << 32), (u64)r.a.z | ((u64)r.a.w << 32), L, N, S, p);
}
__device__ __forceinline__ bool decode_any(const Rec32 &r, int L, int N, int &S, P16 &p) {
  return decode_record_w(r.a, r.b, L, N, S, p);
}
// every stage has exactly one worker (sum of the stage masks' bits = S)
__device__ __forceinline__ bool all_single(const P8 &p, int S) { return __popcll(p.masks) == S; }
__device__ __forceinline__ bool all_single(const P16 &p, int S) {
  return __popcll(p.m[0]) + __popcll(p.m[1]) + __popcll(p.m[2]) + __popcll(p.m[3]) == S;
}
__device__ __forceinline__ const P8 &cur_part(const CurPart &c, const P8 *) { return c.p8; }
__device__ __forceinline__ const P16 &cur_part(const CurPart &c, const P16 *) { return c.p16; }

// Round-robin replicas (row f4): the recurrence for up to q.rounds rounds (RR_DEFER_ROUNDS); a record whose
// bounds have not met by then goes to the deferral queue with its bracket (its T is written by the
// drain kernel), or, when the queue is full, is finished here.
__device__ __forceinline__ u64 rr_eval(const SmemTab &t, int S, const P8 &p, int sync, u64 i, const RRQueue &q) {
  if (!q.buf) return rr_time(t, S, p, sync);
  // one worker per stage: the split model's closed form (reading F-5, C-2 the case r = 1)
  if (__popcll(p.masks) == S) return eval_closed_form<false, false, P8>(t, S, p, sync);
  RRSetup R;
  rr_setup(t, S, p, sync, R);
  if (S == 1) return umax(rr_single_stage(R), R.Tsync);
  u64 t_lo, t_hi;
  if (rr_sim(R, q.rounds, U64MAX, t_lo, t_hi, nullptr) == RR_MET || R.Tsync >= t_hi) return umax(t_lo, R.Tsync);
  const u32 k = atomicAdd(q.n, 1u);
  if (k < q.cap) {
    q.buf[3 * (u64)k] = i;
    q.buf[3 * (u64)k + 1] = t_lo;
    q.buf[3 * (u64)k + 2] = t_hi;
    return U64MAX;  // overwritten by k_rr_drain
  }
  return umax(rr_ceil_bf(R, t_lo, t_hi), R.Tsync);
}
template <typename P>
__device__ __forceinline__ u64 rr_eval(const SmemTab &, int, const P &, int, u64, const RRQueue &) {
  return U64MAX;  // wide records: refused by the host
}

// The 32-bit F + B prefix is staged for the r = 1 closed form of 16-byte records under PipeDream on a
// 32-bit or narrow state (launch_eval sizes the dynamic shared memory to match).
template <int MODE, bool P32, bool NARROW, typename P>
struct PCT {
  static constexpr bool value = MODE == SCHED_PIPEDREAM && P::MS == 8 && (P32 || NARROW);
};

// Scores the record in `slot` and overwrites the slot with its results (bytes 0..7: T, 8..15: switch
// bytes); the traversal then stores the chunk's results in input order, coalesced.
template <bool ROLLOUT, bool P32, int MODE, bool NARROW, typename P, typename Rec>
__device__ __forceinline__ void score_one(const SmemTab &t, int L, int N, bool overflow, Rec &slot,
                                          const CurPart &cur, const ModelP &m, u64 i, const RRQueue &q) {
  int S;
  P p;
  u64 T = U64MAX, sw = U64MAX;
  const bool ok = !overflow && decode_any(slot, L, N, S, p);
  // the lean r = 1 closed form when every active lane holds a one-worker-per-stage record (the
  // shape sort puts them together); a mixed step keeps the general form, so lanes do not diverge
  const bool lean = MODE == SCHED_PIPEDREAM && __all_sync(__activemask(), ok && all_single(p, S));
  if (ok) {
    if (lean) T = eval_r1<P32, NARROW, P, PCT<MODE, P32, NARROW, P>::value>(t, S, p);
    else if constexpr (MODE == SCHED_RR) T = rr_eval(t, S, p, (int)m.sync, i, q);
    else if constexpr (NARROW) T = eval_closed_form_n<P32, P>(t, S, p, (int)m.sync);
    else T = model_time<MODE, P32>(t, S, p, m);
    if (ROLLOUT) sw = switch_bytes(t, S, p, cur.S, cur_part(cur, (const P *)nullptr));
  }
  slot.a = make_uint4((u32)T, (u32)(T >> 32), (u32)sw, (u32)(sw >> 32));
}

// MODE: the schedule of the model (row f3; SCHED_PIPEDREAM is the 1F1B closed form of rows a4-a7).
// Rec / P: 16-byte records (P8) or 32-byte wide records (P16, row f4).
// NARROW (PipeDream only): the 32-bit stage and shard arithmetic of eval_closed_form_n (status bit 2)
template <bool ROLLOUT, bool P32, int MODE, typename Rec, typename P, bool NARROW = false>
__global__ void __launch_bounds__(EVAL_NT, EVAL_BLOCKS(MODE, P))
    k_eval(DevTables g, const Rec *__restrict__ recs, u64 count, u64 *__restrict__ out_t, u64 *__restrict__ out_sw,
           CurPart cur, ModelP m, u32 *counter, RRQueue rrq) {
  extern __shared__ u64 sm[];
  const SmemTab t = stage_tables<NARROW, PCT<MODE, P32, NARROW, P>::value>(g, sm);
  const int L = t.L, N = (int)g.N;
  // a state that failed the device-side overflow check (set_state_device) scores nothing
  const bool overflow = (g.status[0] & 1ull) != 0;
  for_each_sorted_warp<EVAL_NT / 32, Rec, MODE == SCHED_RR>(
      recs, count, counter,
      [&](Rec &slot, u64 i) { score_one<ROLLOUT, P32, MODE, NARROW, P>(t, L, N, overflow, slot, cur, m, i, rrq); },
      [&](const Rec &slot, u64 i) {
        out_t[i] = (u64)slot.a.x | ((u64)slot.a.y << 32);
        if (ROLLOUT) out_sw[i] = (u64)slot.a.z | ((u64)slot.a.w << 32);
      });
}

// Drain of the round-robin deferral queue: a warp per queued record re-derives its setup and decides
// ceil(lambda) inside the recorded bracket by warp-parallel Bellman-Ford passes over the one-period
// event graph (rr.cuh), then writes T. Grid: one block of 8 warps per SM, warps striding the queue.
constexpr int RR_DRAIN_NT = 256;
__global__ void __launch_bounds__(RR_DRAIN_NT) k_rr_drain(DevTables g, const Rec16 *__restrict__ recs,
                                                          u64 *__restrict__ out_t, RRQueue q, ModelP m) {
  const u32 n = umin(*q.n, q.cap);
  if (n == 0) return;  // nothing deferred: skip the table staging
  extern __shared__ u64 sm[];
  __shared__ long long dist[RR_DRAIN_NT / 32][RR_BF_NODES];
  const SmemTab t = stage_tables<false>(g, sm);
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (u32 k = blockIdx.x * (RR_DRAIN_NT / 32) + w; k < n; k += gridDim.x * (RR_DRAIN_NT / 32)) {
    const u64 i = q.buf[3 * (u64)k], t_lo = q.buf[3 * (u64)k + 1], t_hi = q.buf[3 * (u64)k + 2];
    const Rec16 r = load_rec(recs + i);
    int S;
    P8 p;
    decode_any(r, t.L, (int)g.N, S, p);  // valid: it was scored once already
    RRSetup R;
    rr_setup(t, S, p, (int)m.sync, R);
    const u64 T = umax(rr_ceil_bf_warp(R, t_lo, t_hi, dist[w]), R.Tsync);
    if (lane == 0) out_t[i] = T;
    __syncwarp();
  }
}

template <bool ROLLOUT, bool P32, int MODE, typename Rec, typename P, bool NARROW = false>
static void run_eval(int sms, size_t smem, cudaStream_t st, const DevTables &g, const void *recs, u64 count,
                     u64 *out_t, u64 *out_sw, const CurPart &cur, const ModelP &m, u32 *counter,
                     const RRQueue &rrq) {
  auto kern = k_eval<ROLLOUT, P32, MODE, Rec, P, NARROW>;
  // one wave of resident blocks, fewer for a small batch. The dynamic shared memory (state tables)
  // comes on top of the warps' static sort slices, so the opt-in limit is raised once per kernel;
  // the occupancy is cached per dynamic size (a few sizes per process: one per (L, N)).
  static bool attr = false;
  if (!attr) {
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, kern);
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024 - (int)fa.sharedSizeBytes);
    attr = true;
  }
  static size_t c_smem[8] = {0};
  static int c_occ[8] = {0};
  int occ = 0;
  for (int i = 0; i < 8 && c_occ[i]; ++i)
    if (c_smem[i] == smem) occ = c_occ[i];
  if (!occ) {
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, EVAL_NT, smem) != cudaSuccess || occ < 1) occ = 1;
    static int next = 0;
    c_smem[next] = smem;
    c_occ[next] = occ;
    next = (next + 1) % 8;
  }
  constexpr u64 CH = (u64)WarpSort<EVAL_NT / 32, Rec>::CH * (EVAL_NT / 32);  // records per block and round
  const u64 need = (count + CH - 1) / CH;
  const u64 cap = (u64)sms * occ;
  const unsigned grid = (unsigned)(need < cap ? (need ? need : 1) : cap);
  if (!EvalStatic<Rec>::value || MODE == SCHED_RR) cudaMemsetAsync(counter, 0, sizeof(u32), st);
  const bool drain = MODE == SCHED_RR && sizeof(Rec) == 16 && rrq.buf;
  RRQueue q = drain ? rrq : RRQueue();
  if (drain) cudaMemsetAsync(q.n, 0, sizeof(u32), st);
  kern<<<grid, EVAL_NT, smem, st>>>(g, (const Rec *)recs, count, out_t, out_sw, cur, m, counter, q);
  if (drain) {
    static bool dattr = false;
    if (!dattr) {
      cudaFuncAttributes fa;
      cudaFuncGetAttributes(&fa, k_rr_drain);
      cudaFuncSetAttribute(k_rr_drain, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           227 * 1024 - (int)fa.sharedSizeBytes);
      dattr = true;
    }
    k_rr_drain<<<sms, RR_DRAIN_NT, smem, st>>>(g, (const Rec16 *)recs, out_t, q, m);
  }
}

template <bool ROLLOUT, typename Rec, typename P>
static void dispatch_eval(int sms, size_t smem, cudaStream_t st, const DevTables &g, const void *recs, u64 count,
                          u64 *out_t, u64 *out_sw, const CurPart &cur, const ModelP &m, int path32, u32 *ctr,
                          const RRQueue &rrq) {
  switch (m.sched) {
    case SCHED_2BW: run_eval<ROLLOUT, false, SCHED_2BW, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
    case SCHED_GPIPE: run_eval<ROLLOUT, false, SCHED_GPIPE, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
    case SCHED_DAPPLE: run_eval<ROLLOUT, false, SCHED_DAPPLE, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
    case SCHED_RR: run_eval<ROLLOUT, false, SCHED_RR, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
    case SCHED_CHIMERA: run_eval<ROLLOUT, false, SCHED_CHIMERA, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
    default:  // path32: bit 0 = 32-bit segment sums, bit 1 = narrow stage and shard arithmetic
      switch (path32 & 3) {
        case 3: run_eval<ROLLOUT, true, SCHED_PIPEDREAM, Rec, P, true>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
        case 2: run_eval<ROLLOUT, false, SCHED_PIPEDREAM, Rec, P, true>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
        case 1: run_eval<ROLLOUT, true, SCHED_PIPEDREAM, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq); break;
        default: run_eval<ROLLOUT, false, SCHED_PIPEDREAM, Rec, P>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, ctr, rrq);
      }
  }
}

// cur_rec: the current partition's record (16 or 32 bytes as `wide`), already validated by the host,
// or nullptr. Its S and parts are decoded here.
int launch_eval(const DevTables &g, const void *recs, u64 count, bool wide, u64 *out_t, u64 *out_sw,
                const int *cur_S, const u64 *cur_cuts, const u64 *cur_masks, int path32, const ModelP &m, int sms,
                u32 *counter, cudaStream_t st, const RRQueue &rrq) {
  if (count == 0) return 0;
  // + the 32-bit F + B prefix for the PipeDream r = 1 closed form (PCT), when the kernel stages it
  const bool pc = !wide && m.sched == SCHED_PIPEDREAM && (path32 & 3) != 0;
  const size_t smem = (size_t)smem_words(g.L, g.N, (path32 & 2) != 0, pc) * sizeof(u64);
  CurPart cur;
  memset(&cur, 0, sizeof(cur));
  if (cur_S) {
    cur.S = *cur_S;
    if (wide) {
      cur.p16.c[0] = cur_cuts[0];
      cur.p16.c[1] = cur_cuts[1];
      for (int i = 0; i < 4; ++i) cur.p16.m[i] = cur_masks[i];
    } else {
      cur.p8.cuts = cur_cuts[0];
      cur.p8.masks = cur_masks[0];
    }
    cur.valid = 1;
  }
  if (wide) {
    if (out_sw) dispatch_eval<true, Rec32, P16>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, path32, counter, rrq);
    else dispatch_eval<false, Rec32, P16>(sms, smem, st, g, recs, count, out_t, nullptr, cur, m, path32, counter, rrq);
  } else {
    if (out_sw) dispatch_eval<true, Rec16, P8>(sms, smem, st, g, recs, count, out_t, out_sw, cur, m, path32, counter, rrq);
    else dispatch_eval<false, Rec16, P8>(sms, smem, st, g, recs, count, out_t, nullptr, cur, m, path32, counter, rrq);
  }
  return (m.sched == SCHED_RR && !wide && rrq.buf) ? 2 : 1;
}

}  // namespace ap
