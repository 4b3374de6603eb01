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

__device__ __forceinline__ u64 first_subset(int k) {
  u64 p = 0;
  for (int j = 0; j < k; ++j) p |= (u64)j << (8 * j);
  return p;
}

// masks of a contiguous placement: stage s gets workers [R_{s-1}, R_s)
__device__ __forceinline__ u64 masks_from(const SearchSpace &sp, int S, u64 Rp) {
  const bool all = sp.flags & 1;
  u64 masks = 0;
  int prev = 0;
#pragma unroll
  for (int s = 0; s < MAXS; ++s) {
    if (s < S) {
      const int R = (all && s == S - 1) ? sp.N : byte_at(Rp, s) + 1;
      const u32 m = ((1u << R) - 1u) & ~((1u << prev) - 1u);
      masks |= (u64)m << (8 * s);
      prev = R;
    }
  }
  return masks;
}

__device__ __forceinline__ int comp_k(const SearchSpace &sp, int S) { return (sp.flags & 1) ? S - 1 : S; }
__device__ __forceinline__ int comp_n(const SearchSpace &sp) { return (sp.flags & 1) ? sp.N - 1 : sp.N; }

__device__ __forceinline__ void unrank_global(const SearchSpace &sp, u64 idx, int &S, u64 &Rp, u64 &cuts) {
  S = sp.s_min;
  while (S < sp.s_max && idx >= sp.off[S + 1]) ++S;
  const u64 rem = idx - sp.off[S];
  const u64 rho = rem / sp.ncut[S], kappa = rem % sp.ncut[S];
  Rp = lex_unrank_packed(rho, comp_k(sp, S), comp_n(sp));
  cuts = lex_unrank_packed(kappa, S - 1, sp.L - 1);
}

// same, against a binomial table in shared memory (fixed-length binary searches, no divergence)
__device__ __forceinline__ void unrank_global_smem(const SearchSpace &sp, u64 idx, int &S, u64 &Rp, u64 &cuts,
                                                   const u64 *Bn) {
  S = sp.s_min;
  while (S < sp.s_max && idx >= sp.off[S + 1]) ++S;
  const u64 rem = idx - sp.off[S];
  const u64 rho = rem / sp.ncut[S], kappa = rem % sp.ncut[S];
  Rp = lex_unrank_smem(rho, comp_k(sp, S), comp_n(sp), Bn);
  cuts = lex_unrank_smem(kappa, S - 1, sp.L - 1, Bn);
}

template <int NT, bool P32, int MODE>
__global__ void __launch_bounds__(NT) k_search_generic(DevTables g, SearchSpace sp, u64 begin, u64 end,
                                                       u64 per_thread, BlockOut *out, ModelP m) {
  extern __shared__ u64 sm[];
  // binomial rows n <= L (n = N <= 8 <= L + 1 for the compositions too) after the state tables
  u64 *Bn = sm + smem_words(g.L, g.N);
  const int nb = ((int)g.L + 1 > 9 ? (int)g.L + 1 : 9) * BINOM_K;
  for (int i = threadIdx.x; i < nb; i += NT) Bn[i] = c_binom[i / BINOM_K][i % BINOM_K];
  const SmemTab t = stage_tables(g, sm);  // ends with __syncthreads()
  const u64 gtid = (u64)blockIdx.x * NT + threadIdx.x;
  u64 bestT = U64MAX, bestI = U64MAX, cnt = 0;
  const u64 span = end - begin;
  if (gtid < (span + per_thread - 1) / per_thread) {
    const u64 i0 = begin + gtid * per_thread;
    const u64 i1 = (end - i0 < per_thread) ? end : i0 + per_thread;
    int S;
    u64 Rp, cuts;
    unrank_global_smem(sp, i0, S, Rp, cuts, Bn);
    u64 masks = masks_from(sp, S, Rp);
    for (u64 i = i0; i < i1; ++i) {
      const u64 T = model_time<MODE, P32>(t, S, cuts, masks, m);
      if (T < bestT) {  // indices increase along the thread's range: strict < keeps the first
        bestT = T;
        bestI = i;
      }
      ++cnt;
      if (i + 1 == i1) break;
      if (!lex_next_packed(cuts, S - 1, sp.L - 1)) {  // cut set exhausted: next composition
        cuts = first_subset(S - 1);
        if (!lex_next_packed(Rp, comp_k(sp, S), comp_n(sp))) {  // compositions exhausted: next S
          ++S;
          if (S > sp.s_max) break;
          Rp = first_subset(comp_k(sp, S));
          cuts = first_subset(S - 1);
        }
        masks = masks_from(sp, S, Rp);
      }
    }
  }
  block_minloc_store<NT>(bestT, bestI, cnt, out + blockIdx.x);
}

int launch_search_generic(const DevTables &g, const SearchSpace &sp, u64 begin, u64 end, int path32, const ModelP &m,
                          int sms, BlockOut *out, int max_blocks, int *nblocks, cudaStream_t st) {
  constexpr int NT = 256;
  const u64 span = end - begin;
  // at least 4 candidates per thread (the unrank is a few binary searches); up to 8 blocks per SM.
  // A flushed schedule costs ~M S stage steps per candidate: one candidate per thread is enough.
  const u64 min_per = (m.sched == SCHED_GPIPE || m.sched == SCHED_DAPPLE) ? 1 : 4;
  u64 threads = (span + min_per - 1) / min_per;
  u64 blocks = (threads + NT - 1) / NT;
  const u64 cap = (u64)sms * 8 < (u64)max_blocks ? (u64)sms * 8 : (u64)max_blocks;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  const u64 per = (span + blocks * NT - 1) / (blocks * NT);
  const size_t smem = ((size_t)smem_words(g.L, g.N) + (size_t)((g.L + 1 > 9 ? g.L + 1 : 9) * BINOM_K)) * sizeof(u64);
  const unsigned nbk = (unsigned)blocks;
  const u64 pt = per ? per : 1;
  switch (m.sched) {
    case SCHED_2BW: k_search_generic<NT, false, SCHED_2BW><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m); break;
    case SCHED_GPIPE: k_search_generic<NT, false, SCHED_GPIPE><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m); break;
    case SCHED_DAPPLE: k_search_generic<NT, false, SCHED_DAPPLE><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m); break;
    default:
      if (path32) k_search_generic<NT, true, SCHED_PIPEDREAM><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m);
      else k_search_generic<NT, false, SCHED_PIPEDREAM><<<nbk, NT, smem, st>>>(g, sp, begin, end, pt, out, m);
  }
  *nblocks = (int)blocks;
  return 1;
}

// ---------------------------------------------------------------------------------------------
// grid-level finalisation: one block reduces the per-block (T, index, count) entries, then decodes
// the winning index into its 16-byte partition record.
// ---------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_finalize(const BlockOut *in, int n, SearchSpace sp, ResultDev *res) {
  // binomial rows 0..L (all the unranking needs) in shared memory: the winner is decoded with
  // fixed-length binary searches instead of a serial walk over __constant__ (which misses its cache)
  __shared__ u64 Bn[(MAXL + 1) * BINOM_K];
  const int rows = (sp.L > sp.N ? sp.L : sp.N) + 1;  // cut sets of {0..L-2}, compositions of {1..N}
  for (int i = threadIdx.x; i < rows * BINOM_K; i += 256) Bn[i] = c_binom[i / BINOM_K][i % BINOM_K];
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
    unsigned char rec[16];
    for (int i = 0; i < 16; ++i) rec[i] = 0xFF;
    if (slot.idx != U64MAX) {
      int S;
      u64 Rp, cuts;
      unrank_global_smem(sp, slot.idx, S, Rp, cuts, Bn);
      const u64 masks = masks_from(sp, S, Rp);
      rec[0] = (unsigned char)S;
      for (int s = 0; s < S - 1; ++s) rec[1 + s] = (unsigned char)byte_at(cuts, s);
      for (int s = 0; s < S; ++s)
        for (int w = 0; w < MAXN; ++w)
          if ((byte_at(masks, s) >> w) & 1) rec[8 + w] = (unsigned char)s;
    }
    for (int i = 0; i < 16; ++i) res->part[i] = rec[i];
  }
}

int launch_finalize(const BlockOut *in, int n, const SearchSpace &sp, ResultDev *out, cudaStream_t st) {
  k_finalize<<<1, 256, 0, st>>>(in, n, sp, out);
  return 1;
}

}  // namespace ap
