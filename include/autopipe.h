/*
 * autopipe.h — C-ABI of the B200-native AutoPipe partition cost-model engine.
 *
 * The operation is the pipeline cost model of AutoPipe (Hu, Liu, Wang, Wang; ICPP '24) that scores
 * worker partitions: for a per-layer profile (Table 1 rows L, O, G, P) and a
 * cluster state (Table 1 rows N, B, FP, BP) it returns, in integer nanoseconds,
 * the exact steady-state time per mini-batch of a PipeDream-style 1F1B pipeline (PAPER.md:253-278,
 * Fig. 2 at 463-475): per-stage compute, p2p activations and input gradients at each boundary
 * (PAPER.md:489-494), ring all-reduce of replicated stages and the
 * pipeline-fill recurrence (Observation 3). SPEC.md fixes every rounding rule;
 * results are bit-exact against the CPU oracle in oracle/.
 *
 * Conventions (all functions):
 *  - return AUTOPIPE_OK (0) on success or a negative AUTOPIPE_E_* code; autopipe_last_error(ctx)
 *    then returns a static, NUL-terminated description (valid until the next call on ctx);
 *  - "host pointer" = ordinary CPU memory, read during the call and never retained;
 *    "device pointer" = memory of ctx's CUDA device (e.g. a torch tensor's data_ptr()), which must
 *    stay valid until the work enqueued on `stream` has completed;
 *  - `stream` is a cudaStream_t passed as void* (NULL = the legacy default stream);
 *  - a context is bound to one CUDA device and is not thread-safe; use one per thread/device;
 *  - there is no CPU fallback: every score is computed by the sm_100a kernels of this library.
 */
#ifndef AUTOPIPE_H_
#define AUTOPIPE_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  AUTOPIPE_OK = 0,
  AUTOPIPE_E_INVAL = -1,    /* bad argument (range, NULL pointer, invalid current partition) */
  AUTOPIPE_E_STATE = -2,    /* called in the wrong order (no profile, or no state since the profile) */
  AUTOPIPE_E_OVERFLOW = -3, /* inputs whose exact integer arithmetic would not fit (SPEC.md §7) */
  AUTOPIPE_E_CUDA = -4,     /* a CUDA runtime error (message carries cudaGetErrorString) */
  AUTOPIPE_E_NOMEM = -5     /* device or host allocation failed */
};

/* search flags */
#define AUTOPIPE_USE_ALL_WORKERS 1u /* only partitions with sum r_s = N (reading C-12); default sum r_s <= N */

#define AUTOPIPE_IDLE 0xFFu
#define AUTOPIPE_MAX_STAGES 8
#define AUTOPIPE_MAX_WORKERS 8
#define AUTOPIPE_MAX_LAYERS 255

typedef struct autopipe_ctx autopipe_ctx; /* opaque */

/* One worker partition ("an array of size N, each element the layers assigned to
 * that worker"), exactly 16 bytes so a kernel reads it with one 128-bit load. */
typedef struct {
  uint8_t n_stages;           /* S in [1, min(8, N)] */
  uint8_t last_layer[7];      /* e_0 < ... < e_{S-2} < L-1 (stage s = layers [e_{s-1}+1, e_s]);
                                 e_{S-1} = L-1 is implied; entries >= S-1 are ignored (write 0xFF) */
  uint8_t stage_of_worker[8]; /* per worker w: its stage in [0, S), or 0xFF when idle; w >= N must be 0xFF */
} autopipe_partition;

/* Result of a search: the lexicographic minimum of (time_ns, index) over the scanned shard. */
typedef struct {
  uint64_t time_ns;         /* T_ns of the best candidate (UINT64_MAX if the shard was empty) */
  uint64_t index;           /* its global index (SPEC.md §5) (UINT64_MAX if empty) */
  uint64_t evaluated;       /* number of candidates whose score was decided (= shard size) */
  autopipe_partition part;  /* the best candidate, decoded */
} autopipe_result;

/* NEXT row f4 — the wide record: up to 16 stages and 16 workers, for clusters beyond 8 GPUs such as
 * the paper's 10-GPU testbed. Same meaning and validity rules as
 * autopipe_partition with S in [1, min(16, N)]; exactly 32 bytes (two 128-bit loads). */
#define AUTOPIPE_MAX_STAGES_W 16
#define AUTOPIPE_MAX_WORKERS_W 16
typedef struct {
  uint8_t n_stages;            /* S in [1, min(16, N)] */
  uint8_t last_layer[15];      /* e_0 < ... < e_{S-2} < L-1; entries >= S-1 ignored (write 0xFF) */
  uint8_t stage_of_worker[16]; /* per worker w: its stage in [0, S), or 0xFF; w >= N must be 0xFF */
} autopipe_partition_w;
typedef struct {
  uint64_t time_ns, index, evaluated;
  autopipe_partition_w part;
} autopipe_result_w;

/* Create a context on CUDA device `cuda_device` (the caller's current device is left unchanged
 * on return). Returns E_INVAL for a NULL `out`, E_CUDA if the device cannot be used. */
int autopipe_create(int cuda_device, autopipe_ctx **out);

/* Release every device and host resource of ctx (NULL is a no-op). Synchronises ctx's device. */
void autopipe_destroy(autopipe_ctx *ctx);

/* Description of the last error on ctx ("" if none). NULL ctx -> description of the last
 * autopipe_create failure. */
const char *autopipe_last_error(const autopipe_ctx *ctx);

/* Static metrics (Table 1 rows L, O_i, G_i, P_i, measured once before training,
 * PAPER.md:819-822). Host pointers, L entries each, copied (the caller keeps ownership):
 *   act_bytes[l]    O[l]  bytes of layer l's output activation (sent forward at a cut after l);
 *   grad_bytes[l]   G[l]  bytes of the gradient w.r.t. layer l's input (sent backward at a cut
 *                         before l; reading C-6);
 *   weight_bytes[l] P[l]  bytes of layer l's weights (all-reduced when its stage is replicated).
 * L in [1, 255]; any byte count >= 2^56 -> E_OVERFLOW. Invalidates the state: autopipe_set_state
 * must be called before any scoring call (else E_STATE). Synchronous. */
int autopipe_load_profile(autopipe_ctx *ctx, uint32_t L, const uint64_t *act_bytes,
                          const uint64_t *grad_bytes, const uint64_t *weight_bytes);

/* Dynamic metrics (Table 1 rows N, B_i, FP_ij, BP_ij, refreshed every iteration,
 * PAPER.md:823-833). Host pointers, copied:
 *   fp_ns, bp_ns      N x L row-major: forward / backward nanoseconds of layer l on worker w;
 *   link_fs_per_byte  N x N row-major: inverse bandwidth of the directed link u -> v in
 *                     femtoseconds per byte (the per-link form of B_i, reading C-5; the diagonal
 *                     is ignored; 0 = free link).
 * N in [1, 16] (N > 8 is the wide range of row f4: the 16-byte calls then score records naming
 * workers < 8 only, and the 16-byte search / decode / neighbourhood / switch calls return E_INVAL; use
 * the _w calls). Rejects (E_OVERFLOW) states whose products bytes*tau reach 2^64 or whose largest
 * modelled sum reaches 2^59 (SPEC.md §7; the bound counts 7 stage boundaries for N <= 8, 15 for
 * N > 8); picks the 32-bit search path when every r=1 sum fits.
 * Enqueues the prefix-sum and link-table kernels on `stream` (returns before they finish).
 * Requires a loaded profile (E_STATE). */
int autopipe_set_state(autopipe_ctx *ctx, uint32_t N, const uint64_t *fp_ns, const uint64_t *bp_ns,
                       const uint64_t *link_fs_per_byte, void *stream);

/* Same as autopipe_set_state, with the three arrays in DEVICE memory (e.g. written by an on-GPU
 * profiler): nothing is copied from the host. The overflow rules are checked by the state kernel on
 * the device; a violating state makes every later score UINT64_MAX and the next synchronous call
 * (autopipe_search_optimum, autopipe_int_path) reports AUTOPIPE_E_OVERFLOW. The arrays must stay
 * valid until the enqueued kernel has run. Async on `stream`. */
int autopipe_set_state_device(autopipe_ctx *ctx, uint32_t N, const uint64_t *d_fp_ns, const uint64_t *d_bp_ns,
                              const uint64_t *d_link_fs_per_byte, void *stream);

/* Batched scoring of explicit partitions (device pointers; async on `stream`):
 *   d_parts[count]    input records (any disjoint worker sets, reading C-11);
 *   d_time_ns[count]  output T_ns per record; an invalid record (SPEC.md §2) gets UINT64_MAX and
 *                     never fails the batch.
 * count = 0 is a no-op. Requires a state (E_STATE). */
int autopipe_eval_partitions(autopipe_ctx *ctx, const autopipe_partition *d_parts, uint64_t count,
                             uint64_t *d_time_ns, void *stream);

/* Exhaustive search (PAPER.md:896-899 enumerates candidates and scores each with the speed model;
 * here every candidate is scored exactly). Candidates: S in [s_min, s_max] (1 <= s_min <= s_max <=
 * min(8, N)), contiguous worker placement (stage s gets workers [R_{s-1}, R_s)), every cut set;
 * flags: AUTOPIPE_USE_ALL_WORKERS or 0. Scans the global indices [begin, end) of SPEC.md §5
 * (end = UINT64_MAX means "to the end"; end is clamped to the space size), so a space can be split
 * across GPUs or resumed. Writes the shard's lexicographic (time_ns, index) minimum to the host
 * struct *h_out. Synchronous (waits for `stream`). */
int autopipe_search_optimum(autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                            uint64_t begin, uint64_t end, autopipe_result *h_out, void *stream);

/* The same search, asynchronous: the result is written to the DEVICE struct *d_out on `stream` and
 * the call returns once the kernels are enqueued (it waits for the device only when the context's
 * previous search has not yet consumed its schedule copy, and for a schedule other than PipeDream
 * whose state was set from device memory). For a state set with autopipe_set_state_device the host
 * does not read the state back: the kernels of both integer paths are enqueued and each runs only if
 * the state kernel chose its path, so an overflowing device state yields evaluated = 0 and
 * time_ns = index = UINT64_MAX for a non-empty shard (the next synchronous call reports
 * E_OVERFLOW). An empty shard writes (UINT64_MAX, UINT64_MAX, 0, 0xFF...). The context's scratch is
 * shared by its calls: issue a context's asynchronous searches on one stream (or order them).
 * This is the per-rank step of the multi-GPU search (row e): gather the ranks' results and reduce
 * them with autopipe_reduce_results, with no host round trip. */
int autopipe_search_optimum_async(autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                  uint64_t begin, uint64_t end, autopipe_result *d_out, void *stream);

/* Row e, cross-shard bound (north star: "split the index space ... NCCL min-loc"). A shard's sweep
 * filters its candidates against the best T known so far; alone it only knows its own shard, and a
 * shard far from the optimum filters poorly. The bound lets every shard start from the best seed of
 * ALL shards:
 *   1. autopipe_search_seed_async: d_theta (DEVICE u64, caller-owned) is set to UINT64_MAX, then for
 *      every r = 1 block of [begin, end) with >= 2^26 candidates (the blocks whose sweep seeds
 *      itself) the seed kernel's exact T of one candidate of the shard is min-folded into it.
 *      No sweep, no result; asynchronous on `stream`. Blocks with fewer candidates, other S and
 *      other schedules leave it untouched.
 *   2. the caller min-reduces d_theta over the ranks (NCCL all_reduce MIN, 8 bytes);
 *   3. autopipe_set_search_bound(ctx, d_theta): the context's later searches start every r = 1
 *      sweep from theta = *d_theta (read on the device when the sweep starts) instead of running
 *      their own seed; NULL clears it. The pointer must stay valid while it is set. The bound is
 *      keyed to the context's last seed call: it applies only to searches with that call's
 *      (s_min, s_max, flags) while the profile, state and schedule are unchanged (any
 *      load_profile / set_state[_device] / set_schedule retires it, and such searches run
 *      unbounded). E_STATE if the context has no seed call on its current state.
 * A search under a bound returns the shard's exact (time_ns, index) minimum whenever that minimum
 * is <= *d_theta; otherwise its result is (UINT64_MAX, UINT64_MAX, evaluated, 0xFF...) or a
 * candidate with time_ns > *d_theta. Because *d_theta is the exact T of a real candidate of some
 * shard (candidates are still decided one by one, non-strictly against the bound, so ties keep
 * their lowest index), the reduction over all shards (autopipe_reduce_results) is the exact
 * optimum of the whole space, identical to the unbounded search. Errors: E_INVAL (NULL pointer),
 * E_STATE, the argument checks of autopipe_search_optimum. */
int autopipe_search_seed_async(autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                               uint64_t begin, uint64_t end, uint64_t *d_theta, void *stream);
int autopipe_set_search_bound(autopipe_ctx *ctx, const uint64_t *d_bound);

/* Row e (north star: "only a tiny NCCL min-loc allreduce"): d_in[n] results (e.g. all-gathered from
 * the ranks' asynchronous searches; device memory) -> *d_out = their lexicographic (time_ns, index)
 * minimum, evaluated = the sum, the record of the winner (on exact ties, the lowest entry's). Async on
 * `stream`; one warp. n = 0 writes an empty result. Needs no context. */
int autopipe_reduce_results(const autopipe_result *d_in, uint32_t n, autopipe_result *d_out, void *stream);

/* RL rollout rewards (the arbiter sees the current and the new partition; the
 * reward is one-iteration speed with a switching cost). Device pointers, async on `stream`:
 *   d_parts[count]         proposals; d_time_ns[count] gets T_ns (UINT64_MAX if invalid);
 *   h_current              HOST pointer to the current partition, or NULL;
 *   d_switch_bytes[count]  if h_current != NULL: sum over layers l of P[l] * |W_new(l) \ W_old(l)|
 *                          (SPEC.md §6; UINT64_MAX for an invalid proposal); must be NULL when
 *                          h_current is NULL.
 * An invalid *h_current -> E_INVAL. */
int autopipe_rollout_rewards(autopipe_ctx *ctx, const autopipe_partition *d_parts, uint64_t count,
                             const autopipe_partition *h_current, uint64_t *d_time_ns,
                             uint64_t *d_switch_bytes, void *stream);

/* NEXT row f1 — the two-worker neighbourhood ("we limit the new partition solution
 * to only change the two workers' tasks in comparison to the old one"; the partition is the
 * per-worker array of assigned layers). Reading F-1: the neighbourhood
 * of *h_current is every valid partition whose per-worker layer-set array differs from the current
 * one in one or two entries (a worker joining/leaving a stage, a boundary moved between two workers'
 * stages, a stage split between two workers, two workers exchanging stages, ...).
 *   autopipe_neighbourhood: writes the neighbours (canonical records, deterministic order) to the
 *     device array d_out[capacity] and their number to *h_count (which may exceed capacity: only the
 *     first `capacity` are written). Synchronous.
 *   autopipe_neighbourhood_best: scores every neighbour with the cost model and returns the minimum
 *     of (time_ns, record bytes) in *h_out (index = UINT64_MAX, evaluated = neighbourhood size;
 *     time_ns = UINT64_MAX if the neighbourhood is empty). Synchronous.
 * An invalid *h_current -> E_INVAL; requires a state (E_STATE). */
int autopipe_neighbourhood(autopipe_ctx *ctx, const autopipe_partition *h_current, autopipe_partition *d_out,
                           uint64_t capacity, uint64_t *h_count, void *stream);
/* The paper's gradual migration ("gradually migrate ... to the best neighbour"):
 * from *h_start, repeatedly move to the best two-worker neighbour (autopipe_neighbourhood_best)
 * while it is strictly faster, at most max_steps moves. h_path[capacity] (HOST) receives the path:
 * entry 0 = the start (its T_ns, evaluated = 1), then one entry per move (T_ns, evaluated =
 * neighbourhood size, the record); *h_count = entries written. Synchronous; every score comes from
 * the kernels. Errors as autopipe_neighbourhood_best; E_INVAL for NULL pointers or capacity 0. */
int autopipe_local_search(autopipe_ctx *ctx, const autopipe_partition *h_start, uint32_t max_steps,
                          autopipe_result *h_path, uint32_t capacity, uint32_t *h_count, void *stream);
int autopipe_neighbourhood_best(autopipe_ctx *ctx, const autopipe_partition *h_current, autopipe_result *h_out,
                                void *stream);

/* NEXT row f2 — switching cost as time (a switch pauses training and the
 * pipeline "requires a restart phase, i.e., startup starts in Figure 2, which brings bubbles";
 * layer weights move to the workers that newly hold them; the
 * reward is one-iteration speed with the normalised switching cost). Reading F-2:
 *   refill_ns   = max(0, C_{S-1} - S * T_ns): C_k is when stage 0 finishes the backward pass of
 *                 mini-batch k in the 1F1B schedule of the proposal started empty at time 0;
 *   migrate_ns  = max over workers w of the sum of w's weight messages: for every stage of the
 *                 current partition that covers some of w's new layers and does not contain w, one
 *                 message of those layers' weight bytes from the holder with the smallest tau[u][w];
 *   reward_ns   = T_ns + ceil((refill_ns + migrate_ns) / horizon);
 *   both costs are 0 when every worker keeps its layer set (then reward_ns = T_ns).
 * Device pointers, async on `stream`: d_parts[count] proposals; d_reward_ns[count] required;
 * d_time_ns, d_refill_ns, d_migrate_ns may each be NULL. An invalid proposal gets UINT64_MAX in
 * every output. h_current: HOST pointer, required (invalid -> E_INVAL); horizon >= 1 (else E_INVAL).
 * E_OVERFLOW if the state's bound on modelled sums (SPEC.md §7) reaches 2^52 ns (startup event times
 * stay below 2^62). For a state set with autopipe_set_state_device this call synchronises `stream`
 * once to read the state's status. */
int autopipe_switch_rewards(autopipe_ctx *ctx, const autopipe_partition *d_parts, uint64_t count,
                            const autopipe_partition *h_current, uint64_t horizon, uint64_t *d_time_ns,
                            uint64_t *d_refill_ns, uint64_t *d_migrate_ns, uint64_t *d_reward_ns, void *stream);

/* NEXT row f4 — the wide calls: the same operations as autopipe_eval_partitions,
 * autopipe_rollout_rewards, autopipe_search_optimum and autopipe_decode_index over 32-byte records
 * (S <= 16 stages, N <= 16 workers), with the same arguments, ownership, ordering (SPEC.md §5 with S up
 * to min(16, N)), error behaviour and schedule setting (row f3). The search's fast r = 1 kernel serves
 * S in [5, 8]; every other S runs the generic kernel. A space larger than 2^64 -> E_OVERFLOW. */
int autopipe_eval_partitions_w(autopipe_ctx *ctx, const autopipe_partition_w *d_parts, uint64_t count,
                               uint64_t *d_time_ns, void *stream);
int autopipe_rollout_rewards_w(autopipe_ctx *ctx, const autopipe_partition_w *d_parts, uint64_t count,
                               const autopipe_partition_w *h_current, uint64_t *d_time_ns,
                               uint64_t *d_switch_bytes, void *stream);
int autopipe_search_optimum_async_w(autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                    uint64_t begin, uint64_t end, autopipe_result_w *d_out, void *stream);
int autopipe_reduce_results_w(const autopipe_result_w *d_in, uint32_t n, autopipe_result_w *d_out, void *stream);
int autopipe_search_optimum_w(autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags, uint64_t begin,
                              uint64_t end, autopipe_result_w *h_out, void *stream);
int autopipe_decode_index_w(const autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                            uint64_t index, autopipe_partition_w *out);

/* NEXT row f3 — schedule variants and the PS synchronisation scheme. The paper contrasts PipeDream's
 * asynchronous 1F1B with the flushing pipelines GPipe (micro-batches, forward recomputation,
 * PAPER.md:279-292) and DAPPLE and with PipeDream-2BW (double-buffered weights,
 * coalesced weight gradients), applies AutoPipe to DAPPLE and 2BW
 * (PAPER.md:1341-1350), and synchronises data parallelism by PS or ring all-reduce
 * (PAPER.md:1081-1082, 1114-1117). Reading F-3 fixes the timing of each:
 *   schedule      AUTOPIPE_SCHED_PIPEDREAM  static 1F1B steady state, sync every mini-batch (default);
 *                 AUTOPIPE_SCHED_2BW        the same steady state, one sync per M micro-batches;
 *                 AUTOPIPE_SCHED_GPIPE      one flushed iteration: F(0..M-1) then B(0..M-1) per worker;
 *                 AUTOPIPE_SCHED_DAPPLE     one flushed iteration in 1F1B order (min(S-s, M) warm-up);
 *                 AUTOPIPE_SCHED_PIPEDREAM_RR  PipeDream's round-robin replicas (row f4, reading F-5,
 *                                   PAPER.md:371-377): a replicated stage takes whole mini-batches in
 *                                   turn (replica k mod r_s), each replica 1F1B with ceil(R_s / r_s) of
 *                                   its own in flight (R_s = workers of stages s..S-1), one transfer per
 *                                   boundary and mini-batch, one sync per r_s mini-batches; M = 1;
 *                                   16-byte records only (N <= 8; wide calls E_INVAL), the state's bound
 *                                   < 2^45 (E_OVERFLOW);
 *                 AUTOPIPE_SCHED_CHIMERA    Chimera's bidirectional pipelines (row f3, reading F-6,
 *                                   PAPER.md:308-314, 1341-1350): one worker per stage; stage s on w_s
 *                                   (down) and on w_{S-1-s} (up); ceil(M/2) micro-batches down,
 *                                   floor(M/2) up, each pipeline in DAPPLE order, a worker's two lists
 *                                   interleaved by readiness (earliest start; ties: lower down stage,
 *                                   then down), the two copies of a stage synchronised after their last
 *                                   backwards; one flushed iteration; 16-byte and wide records; a
 *                                   record with a replicated stage scores UINT64_MAX;
 *   sync          AUTOPIPE_SYNC_RING (default) or AUTOPIPE_SYNC_PS (a parameter server sharded over
 *                 the stage's replicas, each server taking its pushes and pulls one at a time);
 *   micro_batches M >= 1 micro-batches per iteration (must be 1 for PIPEDREAM; <= 65536);
 *   flags         AUTOPIPE_RECOMPUTE (GPipe only: every backward op re-runs the forward).
 * The profile's FP/BP/O/G then describe one micro-batch, and every T_ns returned by
 * autopipe_eval_partitions, autopipe_rollout_rewards, autopipe_search_optimum and
 * autopipe_neighbourhood_best is the time of one iteration (M micro-batches). The setting belongs to
 * the context and survives load_profile / set_state. Scoring calls under a schedule other than
 * PIPEDREAM return E_OVERFLOW when 16 (M + 1) times the state's bound on modelled sums reaches 2^63
 * (for a device state they synchronise `stream` once to read that bound); autopipe_switch_rewards
 * needs the PIPEDREAM schedule (E_STATE otherwise; either sync). Bad values -> E_INVAL. Host-only. */
#define AUTOPIPE_SCHED_PIPEDREAM 0u
#define AUTOPIPE_SCHED_2BW 1u
#define AUTOPIPE_SCHED_GPIPE 2u
#define AUTOPIPE_SCHED_DAPPLE 3u
#define AUTOPIPE_SCHED_PIPEDREAM_RR 4u
#define AUTOPIPE_SCHED_CHIMERA 5u
#define AUTOPIPE_SYNC_RING 0u
#define AUTOPIPE_SYNC_PS 1u
#define AUTOPIPE_RECOMPUTE 1u
#define AUTOPIPE_MAX_MICRO_BATCHES 65536u
int autopipe_set_schedule(autopipe_ctx *ctx, uint32_t schedule, uint32_t sync, uint32_t micro_batches,
                          uint32_t flags);
/* The context's current schedule setting (any output pointer may be NULL). */
int autopipe_get_schedule(const autopipe_ctx *ctx, uint32_t *schedule, uint32_t *sync, uint32_t *micro_batches,
                          uint32_t *flags);

/* Multi-GPU split: G + 1 global indices bounds[0] = 0 < ... <= bounds[G] = space size
 * such that the contiguous shards [bounds[g], bounds[g+1]) of the space (S in [s_min, s_max], flags as
 * in autopipe_search_optimum; L layers, N workers) cost about the same device time: the estimate
 * counts rows and columns of the fast kernel (short rows cost more per candidate), so shards are not
 * equal in candidates. Host-only (no context, no GPU); any split gives the same global optimum.
 * Wide spaces (row f4: N <= 16, s_max <= min(16, N); the index order of autopipe_search_optimum_w)
 * are split the same way (their S > 8 blocks cost as generic-kernel candidates).
 * E_INVAL on bad arguments, E_OVERFLOW if the space exceeds 2^64. */
int autopipe_balanced_shards(uint32_t L, uint32_t N, uint32_t s_min, uint32_t s_max, uint32_t flags, uint32_t G,
                             uint64_t *bounds);
/* The same split with the cost model of the integer path the shards' state runs (int_path = 32 or
 * 64, as autopipe_int_path reports it: the 32-bit sweep's candidates are cheaper against its per-row
 * work, so its shards move their bounds toward the short rows). E_INVAL for another int_path. */
int autopipe_balanced_shards_path(uint32_t L, uint32_t N, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                  uint32_t G, uint32_t int_path, uint64_t *bounds);

/* Number of candidates of a search space (requires a state for L and N); S up to min(16, N). */
int autopipe_count_candidates(const autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                              uint64_t *total);

/* Decode a global index of a search space into its partition record (host utility). */
int autopipe_decode_index(const autopipe_ctx *ctx, uint32_t s_min, uint32_t s_max, uint32_t flags,
                          uint64_t index, autopipe_partition *out);

/* Which integer path the last set_state selected: 32 or 64 (0 if no state). */
int autopipe_int_path(const autopipe_ctx *ctx);

/* Number of kernels this context has launched so far (for launch accounting in benchmarks). */
uint64_t autopipe_kernel_launches(const autopipe_ctx *ctx);

/* Enable (1) / disable (0) device timing of the search kernels: CUDA events recorded on the launch
 * stream around the enumeration kernels of each autopipe_search_optimum (excluding the final
 * reduction and the result copy). */
int autopipe_set_timing(autopipe_ctx *ctx, int enable);

/* Kernel selection of later searches (the result never depends on it; tests use it to exercise each
 * kernel on small spaces). options: 0 = default (a range of at most 2^21 candidates is searched by
 * one dense launch, every candidate's exact T; a PipeDream range of at most 2^28 by one threshold
 * walk; larger ranges are split per S into the r = 1 sweep and the threshold walk),
 * AUTOPIPE_SEARCH_SPLIT = always the per-S split. E_INVAL on unknown bits. */
#define AUTOPIPE_SEARCH_SPLIT 1u
#define AUTOPIPE_SEARCH_NO_R1 2u  /* the r = 1 blocks through the threshold walk instead of the r = 1 sweep */
/* Round-robin replicas (AUTOPIPE_SCHED_PIPEDREAM_RR) evaluations: a record whose schedule is not
 * pinned within a budget of rounds is deferred to a drain kernel (a warp per record, Bellman-Ford in
 * the bracket its simulation gives). RR_DEFER_ALL: a budget of one round (nearly every record takes
 * the drain); RR_NO_DEFER: no deferral (every record finished in its own thread). Results are
 * identical either way. */
#define AUTOPIPE_RR_DEFER_ALL 4u
#define AUTOPIPE_RR_NO_DEFER 8u
int autopipe_set_search_options(autopipe_ctx *ctx, uint32_t options);

/* Device milliseconds of the enumeration kernels of the last timed search (-1 if none); waits for
 * that search's kernels to finish (an asynchronous search returns before they run). */
double autopipe_last_search_ms(const autopipe_ctx *ctx);

/* The enumeration-kernel times (ms) of the timed searches issued since the previous call, oldest
 * first: up to `cap` values into the host array ms[], their number in *count. Waits for those
 * searches. The context keeps the event pairs of its last 64 timed searches; older ones are lost. */
int autopipe_search_times(autopipe_ctx *ctx, double *ms, uint32_t cap, uint32_t *count);

#ifdef __cplusplus
}
#endif

#endif /* AUTOPIPE_H_ */
