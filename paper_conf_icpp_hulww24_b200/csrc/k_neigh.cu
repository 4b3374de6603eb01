// k_neigh.cu — NEXT row f1: the two-worker neighbourhood of the current partition
// and its best member.
//
// "we limit the new partition solution to only change the two workers' tasks in comparison to the
// old one", the partition being the per-worker array of assigned layers
// (PAPER.md:851-853). Reading F-1: a worker's task is its layer set (its stage's interval
// or nothing); the neighbourhood is every valid partition whose per-worker layer-set array differs
// from the current one in one or two entries.
//
// Generation (k_neigh_gen, one thread per changed-worker set D: N singles then C(N,2) pairs): with
// the workers outside D fixed, their stages' intervals E stay; the layers they no longer cover form
// at most two "gaps" (maximal runs of stages held only by D). Every neighbour with changed set D
// covers the gaps exactly with D's new intervals: no gap -> each changed worker goes idle or joins
// an interval of E; one gap g -> a worker takes g (the other idle, joining E, or also g), or the two
// split g at any layer; two gaps -> one each. Every worker of D must actually change, so each
// neighbour is generated exactly once. Slot = item * NEIGH_MAXOPT + option (deterministic order);
// unused slots hold S = 0 (an invalid record, never chosen). The records are then scored by k_eval
// and reduced by k_neigh_best to the minimum (T_ns, record bytes).
#include "eval.cuh"
#include "internal.h"

namespace ap {

// interval packed as (a | e << 8), -1 = idle
__device__ __forceinline__ int iv_make(int a, int e) { return a | (e << 8); }
__device__ __forceinline__ int iv_a(int v) { return v & 0xFF; }
__device__ __forceinline__ int iv_e(int v) { return (v >> 8) & 0xFF; }

// canonical 16-byte record of a per-worker interval array (intervals tile [0, L-1])
__device__ __forceinline__ uint4 build_record(const int (&iv)[MAXN], int N, int L) {
  unsigned char rec[16];
#pragma unroll
  for (int k = 0; k < 16; ++k) rec[k] = 0xFF;
  int start = 0, S = 0;
#pragma unroll
  for (int s = 0; s < MAXS; ++s) {
    if (start <= L - 1) {
      int e = -1;
#pragma unroll
      for (int w = 0; w < MAXN; ++w)
        if (w < N && iv[w] >= 0 && iv_a(iv[w]) == start) e = iv_e(iv[w]);
      if (e >= 0) {
#pragma unroll
        for (int w = 0; w < MAXN; ++w)
          if (w < N && iv[w] >= 0 && iv_a(iv[w]) == start) rec[8 + w] = (unsigned char)s;
        if (e < L - 1) rec[1 + s] = (unsigned char)e;
        start = e + 1;
        S = s + 1;
      }
    }
  }
  rec[0] = (unsigned char)S;
  uint4 r;
  r.x = rec[0] | (rec[1] << 8) | (rec[2] << 16) | ((u32)rec[3] << 24);
  r.y = rec[4] | (rec[5] << 8) | (rec[6] << 16) | ((u32)rec[7] << 24);
  r.z = rec[8] | (rec[9] << 8) | (rec[10] << 16) | ((u32)rec[11] << 24);
  r.w = rec[12] | (rec[13] << 8) | (rec[14] << 16) | ((u32)rec[15] << 24);
  return r;
}

struct NeighCur {
  u64 cuts, sow;  // current partition: packed cuts, stage of worker (0xFF idle)
  int S, L, N, pad;
};

__global__ void k_neigh_gen(NeighCur c, uint4 *slots) {
  const int item = blockIdx.x * blockDim.x + threadIdx.x;
  const int N = c.N, L = c.L, S = c.S;
  const int npairs = N * (N - 1) / 2;
  if (item >= N + npairs) return;
  uint4 *out = slots + (size_t)item * NEIGH_MAXOPT;
  int i, j = -1;
  if (item < N) {
    i = item;
  } else {  // pair index -> (i, j), i < j, lexicographic
    int k = item - N;
    i = 0;
    while (k >= N - 1 - i) {
      k -= N - 1 - i;
      ++i;
    }
    j = i + 1 + k;
  }
  // current intervals
  int iv[MAXN];
  int st_a[MAXS], st_e[MAXS];
#pragma unroll
  for (int s = 0; s < MAXS; ++s) {
    st_a[s] = (s == 0) ? 0 : byte_at(c.cuts, s - 1) + 1;
    st_e[s] = (s == S - 1) ? L - 1 : byte_at(c.cuts, s);
  }
#pragma unroll
  for (int w = 0; w < MAXN; ++w) {
    const int s = byte_at(c.sow, w);
    iv[w] = (w < N && s < S) ? iv_make(st_a[s < MAXS ? s : 0], st_e[s < MAXS ? s : 0]) : -1;
  }
  const int old_i = iv[i], old_j = (j >= 0) ? iv[j] : -1;
  // covered stages (held by a worker outside D) and the gaps
  bool covered[MAXS];
#pragma unroll
  for (int s = 0; s < MAXS; ++s) {
    covered[s] = false;
#pragma unroll
    for (int w = 0; w < MAXN; ++w)
      if (w < N && w != i && w != j && byte_at(c.sow, w) == s) covered[s] = true;
  }
  int gaps[2] = {-1, -1}, ng = 0;
  int E[MAXS], nE = 0;
  for (int s = 0; s < S; ++s) {
    if (covered[s]) {
      E[nE++] = iv_make(st_a[s], st_e[s]);
    } else {
      const int a = st_a[s];
      int e = st_e[s];
      while (s + 1 < S && !covered[s + 1]) e = st_e[++s];
      if (ng < 2) gaps[ng] = iv_make(a, e);
      ++ng;
    }
  }
  int n = 0;
  auto emit = [&](int ni, int nj) {
    int v[MAXN];
#pragma unroll
    for (int w = 0; w < MAXN; ++w) v[w] = iv[w];
    v[i] = ni;
    if (j >= 0) v[j] = nj;
    out[n++] = build_record(v, N, L);
  };
  if (j < 0) {  // single worker i
    if (ng == 0) {
      if (old_i != -1) emit(-1, 0);
      for (int k = 0; k < nE; ++k)
        if (E[k] != old_i) emit(E[k], 0);
    } else if (ng == 1 && gaps[0] != old_i) {
      emit(gaps[0], 0);
    }
  } else if (ng == 0) {
    for (int a = -1; a < nE; ++a)
      for (int b = -1; b < nE; ++b) {
        const int ni = a < 0 ? -1 : E[a], nj = b < 0 ? -1 : E[b];
        if (ni != old_i && nj != old_j) emit(ni, nj);
      }
  } else if (ng == 1) {
    const int g = gaps[0];
    // (g, x): x idle, joins E, or also g
    for (int b = -2; b < nE; ++b) {
      const int nj = (b == -2) ? -1 : (b == -1) ? g : E[b];
      if (g != old_i && nj != old_j) emit(g, nj);
    }
    // (x, g): x idle or joins E
    for (int a = -1; a < nE; ++a) {
      const int ni = a < 0 ? -1 : E[a];
      if (ni != old_i && g != old_j) emit(ni, g);
    }
    // split g at every layer
    const int gl = iv_a(g), gh = iv_e(g);
    for (int cpos = gl; cpos < gh; ++cpos) {
      const int lo = iv_make(gl, cpos), hi = iv_make(cpos + 1, gh);
      if (lo != old_i && hi != old_j) emit(lo, hi);
      if (hi != old_i && lo != old_j) emit(hi, lo);
    }
  } else if (ng == 2) {
    if (gaps[0] != old_i && gaps[1] != old_j) emit(gaps[0], gaps[1]);
    if (gaps[1] != old_i && gaps[0] != old_j) emit(gaps[1], gaps[0]);
  }
  for (; n < NEIGH_MAXOPT; ++n) out[n] = make_uint4(0, 0, 0, 0);  // S = 0: empty slot
}

// Compaction in slot order + count (one block): the listing API.
__global__ void __launch_bounds__(1024) k_neigh_compact(const uint4 *slots, u64 nslots, uint4 *out, u64 cap,
                                                       u64 *count) {
  __shared__ u64 base;
  __shared__ u32 wsum[32];
  if (threadIdx.x == 0) base = 0;
  __syncthreads();
  for (u64 b = 0; b < nslots; b += 1024) {
    const u64 k = b + threadIdx.x;
    const bool v = k < nslots && (slots[k].x & 0xFF) != 0;
    const u32 bal = __ballot_sync(0xffffffffu, v);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) wsum[wid] = __popc(bal);
    __syncthreads();
    u64 off = base;
    for (int q = 0; q < wid; ++q) off += wsum[q];
    off += __popc(bal & ((1u << lane) - 1));
    if (v && off < cap) out[off] = slots[k];
    __syncthreads();
    if (threadIdx.x == 0) {
      u64 t = 0;
      for (int q = 0; q < 32; ++q) t += wsum[q];
      base += t;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) *count = base;
}

// Minimum of (T, record bytes) over the slots (one block).
__device__ __forceinline__ u64 bytes_be(u64 v) {  // byte 0 most significant: integer order = byte order
  u64 r = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) r = (r << 8) | ((v >> (8 * k)) & 0xFF);
  return r;
}
__device__ __forceinline__ bool key_less(u64 t1, u64 a1, u64 b1, u64 t2, u64 a2, u64 b2) {
  if (t1 != t2) return t1 < t2;
  const u64 A1 = bytes_be(a1), A2 = bytes_be(a2);
  if (A1 != A2) return A1 < A2;
  return bytes_be(b1) < bytes_be(b2);
}

__global__ void __launch_bounds__(1024) k_neigh_best(const uint4 *slots, const u64 *times, u64 nslots,
                                                    ResultDev *res) {
  u64 bt = U64MAX, ba = U64MAX, bb = U64MAX, cnt = 0;
  for (u64 k = threadIdx.x; k < nslots; k += 1024) {
    const uint4 r = slots[k];
    if ((r.x & 0xFF) == 0) continue;
    ++cnt;
    const u64 a = (u64)r.x | ((u64)r.y << 32), b = (u64)r.z | ((u64)r.w << 32);
    if (key_less(times[k], a, b, bt, ba, bb)) {
      bt = times[k];
      ba = a;
      bb = b;
    }
  }
  __shared__ u64 st[32], sa[32], sb[32], sc[32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const u64 t2 = __shfl_xor_sync(0xffffffffu, bt, o), a2 = __shfl_xor_sync(0xffffffffu, ba, o),
              b2 = __shfl_xor_sync(0xffffffffu, bb, o);
    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if (key_less(t2, a2, b2, bt, ba, bb)) { bt = t2; ba = a2; bb = b2; }
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) { st[wid] = bt; sa[wid] = ba; sb[wid] = bb; sc[wid] = cnt; }
  __syncthreads();
  if (threadIdx.x == 0) {
    u64 t = st[0], a = sa[0], b = sb[0], c = sc[0];
    for (int q = 1; q < 32; ++q) {
      c += sc[q];
      if (key_less(st[q], sa[q], sb[q], t, a, b)) { t = st[q]; a = sa[q]; b = sb[q]; }
    }
    res->time_ns = t;
    res->index = U64MAX;
    res->evaluated = c;
    for (int k = 0; k < 8; ++k) {
      res->part[k] = (unsigned char)(a >> (8 * k));
      res->part[8 + k] = (unsigned char)(b >> (8 * k));
    }
  }
}

int launch_neigh_gen(int S, u64 cuts, u64 sow, int L, int N, void *slots, cudaStream_t st) {
  NeighCur c;
  c.cuts = cuts;
  c.sow = sow;
  c.S = S;
  c.L = L;
  c.N = N;
  c.pad = 0;
  const int items = N + N * (N - 1) / 2;
  k_neigh_gen<<<1, 64, 0, st>>>(c, (uint4 *)slots);
  (void)items;
  return 1;
}

int launch_neigh_compact(const void *slots, u64 nslots, void *out, u64 cap, u64 *count, cudaStream_t st) {
  k_neigh_compact<<<1, 1024, 0, st>>>((const uint4 *)slots, nslots, (uint4 *)out, cap, count);
  return 1;
}

int launch_neigh_best(const void *slots, const u64 *times, u64 nslots, ResultDev *res, cudaStream_t st) {
  k_neigh_best<<<1, 1024, 0, st>>>((const uint4 *)slots, times, nslots, res);
  return 1;
}

}  // namespace ap
