// binom.cuh — the combinatorial number system of SPEC.md §5 on the device (rows a3, a8).
// Included once, by kernels.cu (the single device translation unit), which owns c_binom.
#pragma once
#include "common.cuh"

namespace ap {

// Binomial coefficients C(n, k), n < 256, k <= 8, uploaded once per context by autopipe_create.
__constant__ u64 c_binom[BINOM_N][BINOM_K];

void upload_binomials(const u64 (*tab)[BINOM_K]) {
  cudaMemcpyToSymbol(c_binom, tab, sizeof(u64) * BINOM_N * BINOM_K);
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
__device__ __forceinline__ u64 lex_rank_smem(u64 packed, int k, int n, const u64 *B) {
  u64 s = 0;
  for (int i = 0; i < k; ++i) {
    const int c = (int)((packed >> (8 * i)) & 0xFF);
    s += B[(n - 1 - c) * BINOM_K + (k - i)];
  }
  return B[n * BINOM_K + k] - 1 - s;
}

__device__ __forceinline__ u64 lex_unrank_smem(u64 rank, int k, int n, const u64 *B) {
  u64 rp = B[n * BINOM_K + k] - 1 - rank;
  u64 out = 0;
  int hi = n - 1;  // d_i < d_{i-1}
  for (int i = 0; i < k; ++i) {
    const int m = k - i;
    // largest d in [0, hi] with C(d, m) <= rp (C(d, m) is non-decreasing in d)
    int lo = 0, h = hi;
    while (lo < h) {
      const int mid = (lo + h + 1) >> 1;
      if (B[mid * BINOM_K + m] <= rp) lo = mid;
      else h = mid - 1;
    }
    rp -= B[lo * BINOM_K + m];
    out |= (u64)(n - 1 - lo) << (8 * i);
    hi = lo - 1;
  }
  return out;
}

}  // namespace ap
