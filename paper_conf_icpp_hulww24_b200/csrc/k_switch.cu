// k_switch.cu — NEXT row f2: the switching cost of a proposal as time (autopipe_switch_rewards).
//
// The paper's switch pauses training and restarts the pipeline, whose "startup state" (Fig. 2)
// brings bubbles, and moves layer weights to the workers that newly hold them
// (PAPER.md:973-981); the arbiter's reward is the one-iteration time with the normalised switching
// cost. Reading F-2 makes that an integer:
//
//   refill  = max(0, C_{S-1} - S * T)   C_k: stage 0 finishes mini-batch k's backward pass in the
//                                        static 1F1B schedule started empty at time 0
//   migrate = max over workers of the sum of their weight messages (one per old stage that covers
//             some of their new layers without holding them; cheapest holder's link)
//   reward  = T + ceil((refill + migrate) / H)
//
// One thread per proposal. C_{S-1} comes from the schedule's own max-plus recurrence, run round by
// round in dependency order (no event queue):
//   round -1, k = 0..S-1, stages ascending   F_s(k) for k < n_s = S - s
//   round  j = 0..S-1, stages descending      B_s(j), then F_s(j + n_s)
// B_s(j) needs backward boundary s of j, produced just before in the same round by stage s+1;
// F_s(j + n_s) needs forward boundary s-1 of j + n_s, produced one round earlier by stage s-1, so
// one "latest" value per boundary suffices. Every worker keeps its own free time (its op list is
// the 1F1B order), every boundary is a barrier over the sending replicas followed by FIFO transfers
// on its directed links (one per overlapping shard pair; the links of different boundaries are
// distinct, so one free time per pair). Worker state lives in registers (loops over the 8 worker
// slots are unrolled and predicated on the worker's stage); per-pair durations and link free times
// in two small per-thread arrays.
#include "eval.cuh"
#include "internal.h"
#include "sched.cuh"
#include "sortchunk.cuh"

namespace ap {

// The current partition, pre-digested on the host: old stage ranges and per-worker layer sets.
struct SwitchCur {
  u64 wkey;          // byte w: 0xFF idle, else old stage of w
  u32 range[MAXS];   // old stage s: a | e << 8
  u32 wrange[MAXN];  // worker w: a | e << 8, 0xFFFF if idle (its layer set)
  u32 masks[MAXS];   // old stage s: worker bitmask
  int S;
};

// C_{S-1} of the startup (see the file comment). sw: byte w = stage of worker w (0xFF idle).
__device__ __forceinline__ u64 startup_completion(const SmemTab &t, int S, u64 cuts, u64 masks, u64 sw) {
  u64 Fd[MAXN], Bd[MAXN], wf[MAXN];
  int stg[MAXN];
#pragma unroll
  for (int w = 0; w < MAXN; ++w) {
    const int s = byte_at(sw, w);
    stg[w] = s;  // 0xFF never matches a stage
    wf[w] = 0;
    Fd[w] = 0;
    Bd[w] = 0;
    if (s != 0xFF) {
      const int a = (s == 0) ? 0 : byte_at(cuts, s - 1) + 1;
      const int e = (s == S - 1) ? t.L - 1 : byte_at(cuts, s);
      const Div8 dv((u32)__popc((u32)byte_at(masks, s)), t.dv);
      Fd[w] = dv.ceil(t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a]);
      Bd[w] = dv.ceil(t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a]);
    }
  }
  // transfers: one FIFO server per boundary and direction with the boundary's longest transfer (the
  // transfers of a boundary start together at its barrier on links no other boundary uses; see
  // flush_makespan in sched.cuh)
  u64 dF[MAXS], dB[MAXS], lfF[MAXS], lfB[MAXS];
#pragma unroll
  for (int s = 0; s < MAXS; ++s) {
    dF[s] = dB[s] = lfF[s] = lfB[s] = 0;
    if (s < S - 1) {
      const int e = byte_at(cuts, s);
      const u32 ms = (u32)byte_at(masks, s), mn = (u32)byte_at(masks, s + 1);
      boundary_cf_cb<8>(t, e, ms, mn, dF[s], dB[s]);
    }
  }

  u64 fdl[MAXS];  // latest completion of forward boundary s
#pragma unroll
  for (int s = 0; s < MAXS; ++s) fdl[s] = 0;
  // round -1: F_s(k) for k < n_s, k-major so boundary s-1 of k is ready when stage s needs it
  for (int k = 0; k < S; ++k) {
#pragma unroll
    for (int s = 0; s < MAXS; ++s) {
      if (s < S - k) {
        const u64 ready = (s == 0) ? 0 : fdl[s > 0 ? s - 1 : 0];
        u64 bar = 0;
#pragma unroll
        for (int w = 0; w < MAXN; ++w)
          if (stg[w] == s) {
            wf[w] = umax(wf[w], ready) + Fd[w];
            bar = umax(bar, wf[w]);
          }
        if (s < S - 1) {
          lfF[s] = umax(bar, lfF[s]) + dF[s];
          fdl[s] = lfF[s];
        }
      }
    }
  }
  // rounds j = 0..S-1: stages from the last to the first, B_s(j) then F_s(j + n_s)
  u64 C = 0;
  for (int j = 0; j < S; ++j) {
    u64 bd = 0;  // completion of backward boundary s of mini-batch j, flowing towards stage 0
#pragma unroll
    for (int s = MAXS - 1; s >= 0; --s) {
      if (s < S) {
        const u64 readyB = (s == S - 1) ? 0 : bd;
        u64 bar = 0;
#pragma unroll
        for (int w = 0; w < MAXN; ++w)
          if (stg[w] == s) {
            wf[w] = umax(wf[w], readyB) + Bd[w];
            bar = umax(bar, wf[w]);
          }
        if (s > 0) {
          const int sb = s > 0 ? s - 1 : 0;
          lfB[sb] = umax(bar, lfB[sb]) + dB[sb];
          bd = lfB[sb];
        } else {
          C = bar;
        }
        const u64 readyF = (s == 0) ? 0 : fdl[s > 0 ? s - 1 : 0];
        u64 barF = 0;
#pragma unroll
        for (int w = 0; w < MAXN; ++w)
          if (stg[w] == s) {
            wf[w] = umax(wf[w], readyF) + Fd[w];
            barF = umax(barF, wf[w]);
          }
        if (s < S - 1) {
          lfF[s] = umax(barF, lfF[s]) + dF[s];
          fdl[s] = lfF[s];
        }
      }
    }
  }
  return C;
}

// Weight migration (reading F-2): per receiving worker, the sum of its messages; the max over workers.
// tmin[so * 8 + w] = min over the holders u of old stage so of tau[u][w].
__device__ __forceinline__ u64 migrate_time(const SmemTab &t, int S, u64 cuts, u64 sw, const SwitchCur &cur,
                                            const u64 *tmin) {
  u64 best = 0;
#pragma unroll
  for (int w = 0; w < MAXN; ++w) {
    const int s = byte_at(sw, w);
    if (s != 0xFF) {
      const int a = (s == 0) ? 0 : byte_at(cuts, s - 1) + 1;
      const int e = (s == S - 1) ? t.L - 1 : byte_at(cuts, s);
      const int own = byte_at(cur.wkey, w);
      u64 sum = 0;
#pragma unroll
      for (int so = 0; so < MAXS; ++so) {
        if (so < cur.S && so != own) {
          const int lo = max(a, (int)(cur.range[so] & 0xFF)), hi = min(e, (int)(cur.range[so] >> 8));
          if (lo <= hi) sum += xfer(t.PP[hi + 1] - t.PP[lo], tmin[so * 8 + w]);
        }
      }
      best = umax(best, sum);
    }
  }
  return best;
}

#ifndef SWITCH_MINB
#define SWITCH_MINB 2  // B200: 2 blocks per SM (128 registers) beat 1 (171): 1.09 -> 0.82 ms per 1M
#endif
#ifndef SWITCH_SORT
#define SWITCH_SORT 0  // 1: warp-sorted dynamic chunks (sortchunk.cuh), as k_eval
#endif
template <bool P32>
__global__ void __launch_bounds__(256, SWITCH_MINB) k_switch(DevTables g, const uint4 *__restrict__ recs, u64 count,
                                                             SwitchCur cur, u64 horizon, u32 sync, u64 *__restrict__ out_t,
                                                             u64 *__restrict__ out_refill, u64 *__restrict__ out_mig,
                                                             u64 *__restrict__ out_reward, u32 *counter) {
  extern __shared__ u64 sm[];
  const SmemTab t = stage_tables(g, sm);
  __shared__ u64 tmin[MAXS * 8];
  if (threadIdx.x < MAXS * 8) {
    const int so = threadIdx.x >> 3, w = threadIdx.x & 7;
    u64 m = U64MAX;
    if (so < cur.S)
      for (int u = 0; u < MAXN; ++u)
        if ((cur.masks[so] >> u) & 1u) m = umin(m, t.tau[u * TAUW + w]);
    tmin[threadIdx.x] = m;
  }
  __syncthreads();
  const int L = t.L, N = (int)g.N;
  const bool overflow = (g.status[0] & 1ull) != 0;
  auto one = [&](const uint4 &r, u64 i) {
    const u64 lo = (u64)r.x | ((u64)r.y << 32), hi = (u64)r.z | ((u64)r.w << 32);
    int S;
    P8 pp;
    u64 T = U64MAX, R = U64MAX, M = U64MAX, RW = U64MAX;
    if (!overflow && decode_record(lo, hi, L, N, S, pp)) {
      const u64 cuts = pp.cuts, masks = pp.masks;
      T = eval_closed_form<P32>(t, S, pp, (int)sync);
      // per-worker layer sets, compared with the current partition's
      bool same = true;
#pragma unroll
      for (int w = 0; w < MAXN; ++w) {
        const int s = byte_at(hi, w);
        u32 key = 0xFFFFu;
        if (s != 0xFF) {
          const int a = (s == 0) ? 0 : byte_at(cuts, s - 1) + 1;
          const int e = (s == S - 1) ? L - 1 : byte_at(cuts, s);
          key = (u32)a | ((u32)e << 8);
        }
        same &= key == cur.wrange[w];
      }
      if (same) {
        R = 0;
        M = 0;
        RW = T;
      } else {
        const u64 C = startup_completion(t, S, cuts, masks, hi);
        const u64 ST = (u64)S * T;
        R = C > ST ? C - ST : 0;
        M = migrate_time(t, S, cuts, hi, cur, tmin);
        const u64 x = R + M;
        RW = T + (x / horizon + (x % horizon != 0));
      }
    }
    if (out_t) out_t[i] = T;
    if (out_refill) out_refill[i] = R;
    if (out_mig) out_mig[i] = M;
    out_reward[i] = RW;
  };
#if SWITCH_SORT
  for_each_sorted_warp<8>((const Rec16 *)recs, count, counter, [&](const Rec16 &r, u64 i) { one(r.a, i); });
#else
  const u64 stride = (u64)gridDim.x * blockDim.x;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) one(__ldg(recs + i), i);
#endif
}

int launch_switch(const DevTables &g, const void *recs, u64 count, const int cur_S, const u64 cur_cuts,
                  const u64 cur_masks, const u64 cur_sow, u64 horizon, u64 *out_t, u64 *out_refill,
                  u64 *out_mig, u64 *out_reward, int path32, int sync, int sms, u32 *counter, cudaStream_t st) {
  if (count == 0) return 0;
  SwitchCur cur;
  cur.S = cur_S;
  cur.wkey = cur_sow;
  for (int s = 0; s < MAXS; ++s) {
    cur.masks[s] = (u32)((cur_masks >> (8 * s)) & 0xFF);
    cur.range[s] = 0;
    if (s < cur_S) {
      const u32 a = (s == 0) ? 0 : (u32)((cur_cuts >> (8 * (s - 1))) & 0xFF) + 1;
      const u32 e = (s == cur_S - 1) ? g.L - 1 : (u32)((cur_cuts >> (8 * s)) & 0xFF);
      cur.range[s] = a | (e << 8);
    }
  }
  for (int w = 0; w < MAXN; ++w) {
    const int s = (int)((cur_sow >> (8 * w)) & 0xFF);
    cur.wrange[w] = (s == 0xFF) ? 0xFFFFu : cur.range[s];
  }
  const size_t smem = (size_t)smem_words(g.L, g.N) * sizeof(u64);
  const u64 need = (count + 255) / 256, cap = (u64)sms * (SWITCH_SORT ? SWITCH_MINB : 8);
  const int grid = (int)(need < cap ? need : cap);
  if (SWITCH_SORT) {
    static bool attr = false;
    if (!attr) {
      for (auto kern : {k_switch<true>, k_switch<false>}) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, kern);
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024 - (int)fa.sharedSizeBytes);
      }
      attr = true;
    }
    cudaMemsetAsync(counter, 0, sizeof(u32), st);
  }
  if (path32)
    k_switch<true><<<grid, 256, smem, st>>>(g, (const uint4 *)recs, count, cur, horizon, (u32)sync, out_t, out_refill, out_mig,
                                            out_reward, counter);
  else
    k_switch<false><<<grid, 256, smem, st>>>(g, (const uint4 *)recs, count, cur, horizon, (u32)sync, out_t, out_refill, out_mig,
                                             out_reward, counter);
  return 1;
}

}  // namespace ap
