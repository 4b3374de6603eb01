// binom.cuh — the combinatorial number system of SPEC.md §5 on the device (rows a3, a8).
// Included by the search translation units (k_search.cu, k_search_r1.cu); each holds its own copy
// of the tables (internal linkage), filled by upload_binomials (internal.h) at context creation.
#pragma once
#include "common.cuh"

namespace ap {

// Binomial coefficients C(n, k), n < 256, k <= 16 (saturated at UINT64_MAX: a space whose size
// fits 64 bits only ever reads entries below its size), uploaded once per context by autopipe_create.
static __constant__ u64 c_binom[BINOM_N][BINOM_K];
// the same table in global memory, for the kernels that stage rows of it into shared memory: threads
// read different entries, which __constant__ would serialise; global loads coalesce (L2-resident)
static __device__ u64 g_binom[BINOM_N][BINOM_K];

static void upload_binomials_tu(const u64 (*tab)[BINOM_K]) {
  cudaMemcpyToSymbol(c_binom, tab, sizeof(u64) * BINOM_N * BINOM_K);
  cudaMemcpyToSymbol(g_binom, tab, sizeof(u64) * BINOM_N * BINOM_K);
}

// Lexicographic rank of a sorted k-subset {c_0 < ... < c_{k-1}} of {0..n-1} (itertools order):
// rank = C(n,k) - 1 - sum_i C(n-1-c_i, k-i). Subset packed one byte per element, c_0 in byte 0.
__device__ __forceinline__ u64 lex_rank_packed(u64 packed, int k, int n) {
  u64 s = 0;
  for (int i = 0; i < k; ++i) {
    const int c = (int)((packed >> (8 * i)) & 0xFF);
    s += c_binom[n - 1 - c][k - i];
  }
  return c_binom[n][k] - 1 - s;
}

// Inverse of lex_rank_packed: walk each position upward, skipping whole blocks of subsets.
__device__ __forceinline__ u64 lex_unrank_packed(u64 rank, int k, int n) {
  u64 out = 0;
  int x = 0;
  for (int i = 0; i < k; ++i) {
    for (;;) {
      const u64 b = c_binom[n - 1 - x][k - 1 - i];
      if (b > rank) break;
      rank -= b;
      ++x;
    }
    out |= (u64)x << (8 * i);
    ++x;
  }
  return out;
}

// Lexicographic successor of a packed sorted k-subset of {0..n-1}; false when it was the last.
__device__ __forceinline__ bool lex_next_packed(u64 &packed, int k, int n) {
  for (int i = k - 1; i >= 0; --i) {
    const int c = (int)((packed >> (8 * i)) & 0xFF);
    if (c < n - k + i) {
      u64 p = packed & ((i == 0) ? 0ull : ((1ull << (8 * i)) - 1));
      for (int j = i; j < k; ++j) p |= (u64)(c + 1 + (j - i)) << (8 * j);
      packed = p;
      return true;
    }
  }
  return false;
}

// The same two maps against a binomial table held in shared memory (row n = C(n, 0..8)): the hot
// kernel unranks once per lane and task, so it avoids the serialised divergent reads of __constant__.
// Unranking uses the colex dual: r' = C(n,k) - 1 - r = sum_i C(d_i, k-i), d_i = n-1-c_i, each d_i
// found by a fixed-length binary search (no data-dependent trip count, no divergence).
// B: rows n of C(n, 0..BK-1) (BK = BK8 = 9 for 16-byte spaces, BINOM_K = 17 for wide ones).
template <int BK = BK8>
__device__ __forceinline__ u64 lex_rank_smem(u64 packed, int k, int n, const u64 *B) {
  u64 s = 0;
  for (int i = 0; i < k; ++i) {
    const int c = (int)((packed >> (8 * i)) & 0xFF);
    s += B[(n - 1 - c) * BK + (k - i)];
  }
  return B[n * BK + k] - 1 - s;
}

// Byte i of a packed subset: one u64 (k <= 8) or a pair (k <= 16, wide spaces of row f4).
struct Pk2 {
  u64 lo, hi;
};
__device__ __forceinline__ int pk_get(u64 v, int i) { return byte_at(v, i); }
__device__ __forceinline__ int pk_get(const Pk2 &v, int i) { return byte_at(i < 8 ? v.lo : v.hi, i & 7); }
__device__ __forceinline__ void pk_or(u64 &v, int i, int x) { v |= (u64)x << (8 * i); }
__device__ __forceinline__ void pk_or(Pk2 &v, int i, int x) {
  const u64 b = (u64)x << (8 * (i & 7));
  if (i < 8) v.lo |= b;
  else v.hi |= b;
}
__device__ __forceinline__ void pk_zero(u64 &v) { v = 0; }
__device__ __forceinline__ void pk_zero(Pk2 &v) { v.lo = v.hi = 0; }

template <int BK = BK8, typename PK = u64>
__device__ __forceinline__ PK lex_unrank_smem(u64 rank, int k, int n, const u64 *B) {
  u64 rp = B[n * BK + k] - 1 - rank;
  PK out;
  pk_zero(out);
  int hi = n - 1;  // d_i < d_{i-1}
  for (int i = 0; i < k; ++i) {
    const int m = k - i;
    // largest d in [0, hi] with C(d, m) <= rp (C(d, m) is non-decreasing in d)
    int lo = 0, h = hi;
    while (lo < h) {
      const int mid = (lo + h + 1) >> 1;
      if (B[mid * BK + m] <= rp) lo = mid;
      else h = mid - 1;
    }
    rp -= B[lo * BK + m];
    pk_or(out, i, n - 1 - lo);
    hi = lo - 1;
  }
  return out;
}

// Lexicographic successor of a packed sorted k-subset (k <= 16) of {0..n-1}; false when it was the last.
__device__ __forceinline__ bool lex_next_pk2(Pk2 &p, int k, int n) {
  for (int i = k - 1; i >= 0; --i) {
    const int c = pk_get(p, i);
    if (c < n - k + i) {
      Pk2 q;
      // keep bytes 0..i-1, then c+1, c+2, ...
      q.lo = (i >= 8) ? p.lo : (i == 0 ? 0ull : (p.lo & ((1ull << (8 * i)) - 1)));
      q.hi = (i > 8) ? (p.hi & ((1ull << (8 * (i - 8))) - 1)) : 0ull;
      for (int j = i; j < k; ++j) pk_or(q, j, c + 1 + (j - i));
      p = q;
      return true;
    }
  }
  return false;
}

}  // namespace ap
