// internal.h — launchers shared between the host C-ABI (autopipe.cu) and the kernel files.
#pragma once
#include <cuda_runtime.h>
#include "common.cuh"

namespace ap {

// Search space of SPEC.md §5: S in [s_min, s_max], off[S] = global index of the first candidate with
// S stages (off[s_max + 1] = total), ncut[S] = C(L-1, S-1) candidates per composition.
struct SearchSpace {
  int L, N, s_min, s_max, flags, pad0, pad1, pad2;
  u64 off[MAXSW + 2];
  u64 ncut[MAXSW + 2];
  u64 ncomp[MAXSW + 2];
};

// Device-side result of a search (mirrors autopipe_result).
struct ResultDev {
  u64 time_ns, index, evaluated;
  unsigned char part[32];  // the 16-byte record, or the 32-byte wide record (row f4)
};

// Each launcher returns the number of kernels it enqueued (for launch accounting).
int launch_build_state(const DevTables &g, const u64 *fp, const u64 *bp, const u64 *P, const u64 *tau, u64 sumP,
                       cudaStream_t st);
// Explicit records, 16-byte (wide = false) or 32-byte (row f4). cur_cuts / cur_masks: the current
// partition's packed parts (1 and 1 words, or 2 and 4 words for wide), or cur_S = nullptr.
// counter: a device word the launch resets (cudaMemsetAsync) and the kernel's warps draw chunks from.
// path32: bit 0 = the state's 32-bit path, bit 1 = its narrow path (status bit 2; PipeDream only).
// rrq (round-robin replicas only, row f4): the context's deferral queue; records whose schedule has
// not been pinned within RR_DEFER_ROUNDS rounds go there and a drain kernel finishes them, a warp
// per record (k_eval.cu). Without a queue every record is finished in its own thread.
struct RRQueue {
  u64 *buf = nullptr;  // [cap][3]: record index, bracket low, bracket high
  u32 *n = nullptr;    // entries claimed (may exceed cap: those records were finished in the thread)
  u32 cap = 0;
  u32 rounds = 0;      // round budget before a record is deferred
};
#ifndef RR_DEFER_ROUNDS_DEF
#define RR_DEFER_ROUNDS_DEF 256  // B200, 1M C5 records: 128 / 256 / 1024 rounds -> 9.8 / 8.4 / 9.5 ms
#endif
constexpr u32 RR_DEFER_ROUNDS = RR_DEFER_ROUNDS_DEF;
int launch_eval(const DevTables &g, const void *recs, u64 count, bool wide, u64 *out_t, u64 *out_sw,
                const int *cur_S, const u64 *cur_cuts, const u64 *cur_masks, int path32, const ModelP &m, int sms,
                u32 *counter, cudaStream_t st, const RRQueue &rrq = RRQueue());
// Generic exhaustive search over [begin, end) (any S, any composition); writes one BlockOut per block
// into out[out_offset ...] and returns the number of blocks used via *nblocks.
// path32 of a dense launch: bit 0 = 32-bit segment sums, bit 1 = the narrow closed form (-1: gated)
// sched: 32 bytes of device memory the PipeDream launch resets and schedules its chunks through (two
// 16-byte slots: one per gated launch); each concurrent launch needs its own
constexpr int SEARCH_SCHED_BYTES = 32;
int launch_search_generic(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, int path32, const ModelP &m,
                          bool wide, int sms, BlockOut *out, int max_blocks, int *nblocks, void *sched,
                          cudaStream_t st, bool dense = false);
// spaces (or shards) up to this many candidates are searched by one dense launch (one candidate per
// thread, exact T): latency-bound, they finish before a threshold walk would pay off
constexpr unsigned long long DENSE_SPAN = 1ull << 21;
// Cross-shard bound of the r = 1 sweep (row e). bound: device word the sweep's shared theta starts at
// (replaces the shard's own seed); theta_out: seed only, no sweep — the shard's seed T is atomicMin'ed
// into this device word.
struct R1Ext {
  const u64 *bound = nullptr;
  u64 *theta_out = nullptr;
};
// Round-robin replicas search (row f4, 16-byte spaces): the bound-pruned kernel over [begin, end)
// and the drain of its deferred candidates; writes the blocks of both (*nblocks). sched: a 32-byte
// schedule slot; q: the context's deferral queue (not shared with a concurrent launch).
int launch_search_rr(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, const ModelP &m, int sms,
                     BlockOut *out, int max_blocks, int *nblocks, void *sched, const RRQueue &q, cudaStream_t st);
// Fast search over the r = 1 block of one S (all stages on one worker; SPEC.md §5, rho = 0),
// restricted to the cut ranks [k_begin, k_end). path32 selects the 32-bit tables.
int launch_search_r1(const DevTables &g, const SearchSpace &sp, int S, u64 k_begin, u64 k_end,
                     int path32, int sms, BlockOut *out, int max_blocks, int *nblocks, void *work,
                     void *pinned, size_t work_bytes, cudaStream_t st, const R1Ext &ext = R1Ext());
// rec_bytes: record bytes written into out->part (32 for the context's own ResultDev; 16 or 32 when
// out is the caller's autopipe_result / autopipe_result_w)
int launch_finalize(const BlockOut *in, int n, const SearchSpace &sp, ResultDev *out, bool wide, cudaStream_t st,
                    int rec_bytes = 32);
// lexicographic (time_ns, index) minimum of n results of stride 24 + rec_bytes bytes (the autopipe_result
// layout), evaluated counts summed, the winner's record copied (autopipe_reduce_results)
int launch_reduce_results(const void *in, unsigned n, int rec_bytes, void *out, cudaStream_t st);

// the binomial tables of each search translation unit (binom.cuh)
void upload_binomials_search(const u64 (*tab)[BINOM_K]);
void upload_binomials_r1(const u64 (*tab)[BINOM_K]);
inline void upload_binomials(const u64 (*tab)[BINOM_K]) {
  upload_binomials_search(tab);
  upload_binomials_r1(tab);
}

// Tuning knobs for experiments (AUTOPIPE_R1_*, AUTOPIPE_COST_*): read only when the environment sets
// AUTOPIPE_EXPERIMENTS=1; otherwise nullptr, so the production path always runs the measured defaults.
const char *experiment_knob(const char *name);

// NEXT row f1: the two-worker neighbourhood (k_neigh.cu). Slots: (N + C(N,2)) * NEIGH_MAXOPT records.
constexpr int NEIGH_MAXOPT = 544;  // >= (8+2) + (8+1) + 2*(255-1) options per changed-worker set
constexpr int NEIGH_ITEMS = 8 + 28;
int launch_neigh_gen(int S, u64 cuts, u64 sow, int L, int N, void *slots, cudaStream_t st);
int launch_neigh_compact(const void *slots, u64 nslots, void *out, u64 cap, u64 *count, cudaStream_t st);
int launch_neigh_best(const void *slots, const u64 *times, u64 nslots, ResultDev *res, cudaStream_t st);

// NEXT row f2: switching cost as time (k_switch.cu).
int launch_switch(const DevTables &g, const void *recs, u64 count, const int cur_S, const u64 cur_cuts,
                  const u64 cur_masks, const u64 cur_sow, u64 horizon, u64 *out_t, u64 *out_refill,
                  u64 *out_mig, u64 *out_reward, int path32, int sync, int sms, u32 *counter, cudaStream_t st);

}  // namespace ap
