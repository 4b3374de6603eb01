// k_search.cu — exhaustive search (autopipe_search_optimum), rows a3-a8 for the general space:
// combinatorial unranking of the global index (SPEC.md §5), lexicographic successor, the closed form
// per candidate, and a warp -> block -> grid lexicographic (time, index) argmin.
//
// The paper enumerates candidate partitions and scores each with its speed model
// (PAPER.md:896-899); here every candidate of [begin, end) is scored exactly. Launch: a persistent
// grid (a multiple of the SM count) of 256-thread blocks; thread t owns the contiguous index range
// [begin + t*k, begin + (t+1)*k): it unranks its first index once, then steps with the lexicographic
// successor (the last cut moves fastest). Each block writes its (T, index, count); k_finalize reduces
// the blocks and decodes the winner. The argmin is the lexicographic minimum of (T, index), so the
// result does not depend on the grid, the block count or the number of GPUs.
#include "binom.cuh"
#include "eval.cuh"
#include "internal.h"
#include "sched.cuh"

namespace ap {

// Space-generic pieces: a 16-byte space (S, N <= 8: P8, subsets packed in one u64, binomial rows of 9
// columns in shared memory) or a wide one (row f4; S, N <= 16: P16, Pk2 subsets, 17 columns).
template <typename P>
struct SpaceT;
template <>
struct SpaceT<P8> {
  typedef u64 PK;
  static constexpr int BK = BK8;
  __device__ static bool next(PK &p, int k, int n) { return lex_next_packed(p, k, n); }
  __device__ static P8 part(u64 cuts, u64 masks) { return P8{cuts, masks}; }
};
template <>
struct SpaceT<P16> {
  typedef Pk2 PK;
  static constexpr int BK = BINOM_K;
  __device__ static bool next(PK &p, int k, int n) { return lex_next_pk2(p, k, n); }
};

template <typename PK>
__device__ __forceinline__ PK first_subset(int k) {
  PK p;
  pk_zero(p);
  for (int j = 0; j < k; ++j) pk_or(p, j, j);
  return p;
}

__device__ __forceinline__ int comp_k(const SearchSpace &sp, int S) { return (sp.flags & 1) ? S - 1 : S; }
__device__ __forceinline__ int comp_n(const SearchSpace &sp) { return (sp.flags & 1) ? sp.N - 1 : sp.N; }

// The partition of (S, composition Rp, cut set): contiguous placement, stage s gets workers
// [R_{s-1}, R_s) (reading C-11).
template <typename P, typename PK>
__device__ __forceinline__ P part_from(const SearchSpace &sp, int S, const PK &Rp, const PK &cuts) {
  const bool all = sp.flags & 1;
  P p;
  int prev = 0;
  if constexpr (P::MS == 8) {
    p.cuts = cuts;
    p.masks = 0;
  } else {
    p.c[0] = cuts.lo;
    p.c[1] = cuts.hi;
    p.m[0] = p.m[1] = p.m[2] = p.m[3] = 0;
  }
#pragma unroll
  for (int s = 0; s < P::MS; ++s) {
    if (s < S) {
      const int R = (all && s == S - 1) ? sp.N : pk_get(Rp, s) + 1;
      const u32 m = ((1u << R) - 1u) & ~((1u << prev) - 1u);
      if constexpr (P::MS == 8) p.masks |= (u64)m << (8 * s);
      else p.m[s >> 2] |= (u64)m << (16 * (s & 3));
      prev = R;
    }
  }
  return p;
}

// global index -> (S, composition, cut set), against a binomial table in shared memory
// (fixed-length binary searches, no divergence)
template <int BK, typename PK>
__device__ __forceinline__ void unrank_global_smem(const SearchSpace &sp, u64 idx, int &S, PK &Rp, PK &cuts,
                                                   const u64 *Bn) {
  S = sp.s_min;
  while (S < sp.s_max && idx >= sp.off[S + 1]) ++S;
  const u64 rem = idx - sp.off[S];
  const u64 rho = rem / sp.ncut[S], kappa = rem % sp.ncut[S];
  Rp = lex_unrank_smem<BK, PK>(rho, comp_k(sp, S), comp_n(sp), Bn);
  cuts = lex_unrank_smem<BK, PK>(kappa, S - 1, sp.L - 1, Bn);
}

template <int NT, bool P32, int MODE, typename P>
__global__ void __launch_bounds__(NT) k_search_generic(DevTables g, SearchSpace sp, u64 begin, u64 end,
                                                       u64 per_thread, BlockOut *out, ModelP m, int gate) {
  if (gate >= 0 && state_gated_out(g, gate, out)) return;  // see state_gated_out
  typedef SpaceT<P> SP;
  typedef typename SP::PK PK;
  constexpr int BK = SP::BK;
  extern __shared__ u64 sm[];
  // binomial rows n <= L (n = N <= 16 <= L + 1 for the compositions too) after the state tables
  u64 *Bn = sm + smem_words(g.L, g.N);
  const int nb = ((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK;
  for (int i = threadIdx.x; i < nb; i += NT) Bn[i] = g_binom[i / BK][i % BK];
  const SmemTab t = stage_tables(g, sm);  // ends with __syncthreads()
  const u64 gtid = (u64)blockIdx.x * NT + threadIdx.x;
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0;
  const u64 span = end - begin;
  if (gtid < (span + per_thread - 1) / per_thread) {
    const u64 i0 = begin + gtid * per_thread;
    const u64 i1 = (end - i0 < per_thread) ? end : i0 + per_thread;
    int S;
    PK Rp, cuts;
    unrank_global_smem<BK>(sp, i0, S, Rp, cuts, Bn);
    P p = part_from<P>(sp, S, Rp, cuts);
    for (u64 i = i0; i < i1; ++i) {
      const u64 T = model_time<MODE, P32>(t, S, p, m);
      if (T < bestT) {  // indices increase along the thread's range: strict < keeps the first
        bestT = T;
        bestI = i;
      }
      ++cnt;
      if (i + 1 == i1) break;
      if (!SP::next(cuts, S - 1, sp.L - 1)) {  // cut set exhausted: next composition
        cuts = first_subset<PK>(S - 1);
        if (!SP::next(Rp, comp_k(sp, S), comp_n(sp))) {  // compositions exhausted: next S
          ++S;
          if (S > sp.s_max) break;
          Rp = first_subset<PK>(comp_k(sp, S));
          cuts = first_subset<PK>(S - 1);
        }
      }
      p = part_from<P>(sp, S, Rp, cuts);
    }
  }
  block_minloc_store<NT>(bestT, bestI, cnt, out + blockIdx.x);
}

template <int NT, typename P>
static void run_search_generic(unsigned nbk, size_t smem, cudaStream_t st, const DevTables &g, const SearchSpace &sp,
                               u64 begin, u64 end, u64 pt, BlockOut *out, const ModelP &m, int path32) {
  switch (m.sched) {
    case SCHED_2BW: k_search_generic<NT, false, SCHED_2BW, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1); break;
    case SCHED_GPIPE: k_search_generic<NT, false, SCHED_GPIPE, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1); break;
    case SCHED_DAPPLE: k_search_generic<NT, false, SCHED_DAPPLE, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1); break;
    default:
      if (path32 == 1) k_search_generic<NT, true, SCHED_PIPEDREAM, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1);
      else if (path32 == 0) k_search_generic<NT, false, SCHED_PIPEDREAM, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, -1);
      else {  // path chosen on the device (state_gated_out): both, writing disjoint block ranges
        k_search_generic<NT, true, SCHED_PIPEDREAM, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m, 1);
        k_search_generic<NT, false, SCHED_PIPEDREAM, P><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out + nbk, m, 0);
      }
  }
}

int launch_search_generic(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, int path32, const ModelP &m,
                          bool wide, int sms, BlockOut *out, int max_blocks, int *nblocks, cudaStream_t st) {
  constexpr int NT = 256;
  const u64 span = end - begin;
  // at least 4 candidates per thread (the unrank is a few binary searches); up to 8 blocks per SM.
  // A flushed schedule costs ~M S stage steps per candidate: one candidate per thread is enough.
  // A small span (a launch of a short model's space) is latency-bound: one candidate per thread.
  const u64 min_per = (m.sched == SCHED_GPIPE || m.sched == SCHED_DAPPLE || span <= (u64)sms * 8 * NT * 4) ? 1 : 4;
  u64 threads = (span + min_per - 1) / min_per;
  u64 blocks = (threads + NT - 1) / NT;
  const bool both = path32 < 0 && m.sched == SCHED_PIPEDREAM;  // two gated launches share max_blocks
  const u64 room = both ? (u64)max_blocks / 2 : (u64)max_blocks;
  const u64 cap = (u64)sms * 8 < room ? (u64)sms * 8 : room;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  const u64 per = (span + blocks * NT - 1) / (blocks * NT);
  const int BK = wide ? BINOM_K : BK8;
  const size_t smem = ((size_t)smem_words(g.L, g.N) +
                       (size_t)(((int)g.L + 1 > MAXNW + 1 ? (int)g.L + 1 : MAXNW + 1) * BK)) * sizeof(u64);
  const unsigned nbk = (unsigned)blocks;
  const u64 pt = per ? per : 1;
  if (wide) run_search_generic<NT, P16>(nbk, smem, st, g, sp, begin, end, pt, out, m, path32);
  else run_search_generic<NT, P8>(nbk, smem, st, g, sp, begin, end, pt, out, m, path32);
  *nblocks = (int)blocks * (both ? 2 : 1);
  return both ? 2 : 1;
}

// ---------------------------------------------------------------------------------------------
// grid-level finalisation: one block reduces the per-block (T, index, count) entries, then decodes
// the winning index into its partition record (16 bytes, or 32 for a wide space).
// ---------------------------------------------------------------------------------------------
// res: the ResultDev layout (time_ns, index, evaluated, record) with the record cut to rec_bytes (16 or
// 32), so it can be the caller's autopipe_result / autopipe_result_w directly (asynchronous search)
__global__ void __launch_bounds__(256) k_finalize(const BlockOut *in, int n, SearchSpace sp, ResultDev *res, int wide,
                                                 int rec_bytes) {
  // binomial rows 0..L (all the unranking needs) in shared memory: the winner is decoded with
  // fixed-length binary searches instead of a serial walk over __constant__ (which misses its cache)
  __shared__ u64 Bn[(MAXL + 1) * BINOM_K];
  const int BK = wide ? BINOM_K : BK8;
  const int rows = (sp.L > sp.N ? sp.L : sp.N) + 1;  // cut sets of {0..L-2}, compositions of {1..N}
  for (int i = threadIdx.x; i < rows * BK; i += 256) Bn[i] = g_binom[i / BK][i % BK];
  u64 t = U64MAX, idx = U64MAX, cnt = 0;
  for (int i = threadIdx.x; i < n; i += 256) {
    const BlockOut b = in[i];
    if (better(b.t, b.idx, t, idx)) { t = b.t; idx = b.idx; }
    cnt += b.count;
  }
  __shared__ BlockOut slot;
  block_minloc_store<256>(t, idx, cnt, &slot);
  __syncthreads();
  if (threadIdx.x == 0) {
    res->time_ns = slot.t;
    res->index = slot.idx;
    res->evaluated = slot.count;
    unsigned char rec[32];
    for (int i = 0; i < 32; ++i) rec[i] = 0xFF;
    const int off = wide ? 16 : 8;
    if (slot.idx != U64MAX) {
      int S;
      if (wide) {
        Pk2 Rp, cuts;
        unrank_global_smem<BINOM_K>(sp, slot.idx, S, Rp, cuts, Bn);
        const P16 p = part_from<P16>(sp, S, Rp, cuts);
        rec[0] = (unsigned char)S;
        for (int s = 0; s < S - 1; ++s) rec[1 + s] = (unsigned char)p.cut(s);
        for (int s = 0; s < S; ++s)
          for (int w = 0; w < MAXNW; ++w)
            if ((p.mask(s) >> w) & 1) rec[off + w] = (unsigned char)s;
      } else {
        u64 Rp, cuts;
        unrank_global_smem<BK8>(sp, slot.idx, S, Rp, cuts, Bn);
        const P8 p = part_from<P8>(sp, S, Rp, cuts);
        rec[0] = (unsigned char)S;
        for (int s = 0; s < S - 1; ++s) rec[1 + s] = (unsigned char)p.cut(s);
        for (int s = 0; s < S; ++s)
          for (int w = 0; w < MAXN; ++w)
            if ((p.mask(s) >> w) & 1) rec[off + w] = (unsigned char)s;
      }
    }
    for (int i = 0; i < rec_bytes; ++i) res->part[i] = rec[i];
  }
}

int launch_finalize(const BlockOut *in, int n, const SearchSpace &sp, ResultDev *out, bool wide, cudaStream_t st,
                    int rec_bytes) {
  k_finalize<<<1, 256, 0, st>>>(in, n, sp, out, wide ? 1 : 0, rec_bytes);
  return 1;
}

// Row e (multi-GPU): the per-rank search results gathered into one array (an all-gather of
// autopipe_result bytes) reduced to their lexicographic (time_ns, index) minimum, evaluated counts
// summed, the winner's record copied. One warp; n is the number of ranks.
__global__ void k_reduce_results(const unsigned char *in, unsigned n, int rec_bytes, unsigned char *out) {
  const unsigned stride = 24u + (unsigned)rec_bytes;
  u64 t = U64MAX, idx = U64MAX, cnt = 0;
  unsigned who = 0xFFFFFFFFu;
  for (unsigned i = threadIdx.x; i < n; i += 32) {
    const u64 *r = (const u64 *)(in + (size_t)i * stride);
    if (who == 0xFFFFFFFFu || better(r[0], r[1], t, idx)) {  // ascending i: the first of equals stays
      t = r[0];
      idx = r[1];
      who = i;
    }
    cnt += r[2];
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const u64 t2 = __shfl_xor_sync(0xffffffffu, t, o), i2 = __shfl_xor_sync(0xffffffffu, idx, o);
    const unsigned w2 = __shfl_xor_sync(0xffffffffu, who, o);
    // ties on (t, idx) (empty results: both UINT64_MAX) resolve to the lower rank, so the copied record
    // is deterministic
    if (better(t2, i2, t, idx) || (t2 == t && i2 == idx && w2 < who)) { t = t2; idx = i2; who = w2; }
    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  }
  if (threadIdx.x == 0) {
    u64 *o = (u64 *)out;
    o[0] = t;
    o[1] = idx;
    o[2] = cnt;
    const unsigned char *src = in + (size_t)(who == 0xFFFFFFFFu ? 0 : who) * stride + 24;
    for (int b = 0; b < rec_bytes; ++b) out[24 + b] = (n == 0) ? (unsigned char)0xFF : src[b];
  }
}

int launch_reduce_results(const void *in, unsigned n, int rec_bytes, void *out, cudaStream_t st) {
  k_reduce_results<<<1, 32, 0, st>>>((const unsigned char *)in, n, rec_bytes, (unsigned char *)out);
  return 1;
}

void upload_binomials_search(const u64 (*tab)[BINOM_K]) { upload_binomials_tu(tab); }

}  // namespace ap
