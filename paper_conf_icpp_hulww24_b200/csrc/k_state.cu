// k_state.cu — rows a1 and a2: state ingest (per-worker prefix sums of f, b, f+b and of the weight
// bytes), the r = 1 link tables, and the device-side overflow / integer-path check, built on the
// device after every autopipe_set_state / autopipe_set_state_device.
//
// Table 1 inputs: FP_ij, BP_ij (N x L ns), P_i (L bytes), O_i, G_i (L bytes) and
// the per-link inverse bandwidth (reading C-5). One launch, four roles by warp:
//   warps 0 .. 3N   : one row each — warp-shuffle inclusive scan (__shfl_up_sync) over 32-element
//                     chunks with a running carry, written as an exclusive prefix of L + 1 entries
//                     (rows: PF[w], PB[w], PC[w] = prefix of f + b, and PP), plus 32-bit copies of PC;
//   warp 3N + 1     : copies tau (N x N) into the padded 16 x 16 table and computes the overflow /
//                     32-bit-path status of SPEC.md §7 (used when the inputs came from device memory);
//   remaining warps : link tables Z[s][l] = cf + cb and LM[s][l] = max(cf, cb) for the boundary
//                     between worker s and s + 1 at a cut after layer l, with
//                     cf = ceil(O[l] * tau[s][s+1] / 1e6) and cb = ceil(G[l+1] * tau[s+1][s] / 1e6)
//                     (forward activation / backward input gradient, reading C-6), and 32-bit copies.
#include "common.cuh"
#include "internal.h"

namespace ap {

__device__ __forceinline__ u64 warp_incl_scan(u64 v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u64 y = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += y;
  }
  return v;
}

__device__ __forceinline__ u64 warp_max(u64 v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = umax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// fp, bp: [N][L] ns; P: [L] bytes; tau: [N][N] fs/B (any device memory)
__global__ void k_build_state(DevTables g, const u64 *__restrict__ fp, const u64 *__restrict__ bp,
                              const u64 *__restrict__ P, const u64 *__restrict__ tau, u64 sumP, int scan_warps) {
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;  // global warp id
  const int L = (int)g.L, N = (int)g.N, Lp1 = (int)g.Lp1;
  if (gw < scan_warps) {
    // row gw: 0..N-1 -> PF[w], N..2N-1 -> PB[w], 2N..3N-1 -> PC[w], 3N -> PP
    const int kind = gw / N, w = gw % N;
    u64 *dst;
    u32 *dst32 = nullptr;
    if (gw == 3 * N) {
      dst = g.PP;
    } else if (kind == 0) {
      dst = g.PF + w * Lp1;
      dst32 = g.PF32 + w * Lp1;
    } else if (kind == 1) {
      dst = g.PB + w * Lp1;
      dst32 = g.PB32 + w * Lp1;
    } else {
      dst = g.PC + w * Lp1;
      dst32 = g.PC32 + w * Lp1;
    }
    u64 carry = 0;
    if (lane == 0) {
      dst[0] = 0;
      if (dst32) dst32[0] = 0;
    }
    for (int base = 0; base < L; base += 32) {
      const int l = base + lane;
      u64 v = 0;
      if (l < L) {
        if (gw == 3 * N) v = P[l];
        else if (kind == 0) v = fp[w * L + l];
        else if (kind == 1) v = bp[w * L + l];
        else v = fp[w * L + l] + bp[w * L + l];
      }
      const u64 incl = warp_incl_scan(v, lane) + carry;
      if (l < L) {
        dst[l + 1] = incl;
        if (dst32) dst32[l + 1] = (u32)incl;
      }
      carry = __shfl_sync(0xffffffffu, incl, 31);
    }
    return;
  }
  if (gw == scan_warps) {
    // padded tau and the status word (SPEC.md §7 overflow rule, 32-bit search path)
    for (int i = lane; i < TAUW * TAUW; i += 32) {
      const int u = i / TAUW, v = i % TAUW;
      g.tau[i] = (u < N && v < N && u != v) ? tau[u * N + v] : 0ull;
    }
    // ring[mask]: the slowest link of the ring W[0] -> W[1] -> ... -> W[0] over each worker set of up
    // to 8 workers (ascending order; row a6), 0 for sets of fewer than 2
    for (int msk = lane; msk < 256; msk += 32) {
      u64 tr = 0;
      if (__popc(msk) >= 2 && msk < (1 << (N < 8 ? N : 8))) {
        const int first = __ffs(msk) - 1;
        int prev = first;
        int mm = msk & (msk - 1);
        while (mm) {
          const int w = __ffs(mm) - 1;
          mm &= mm - 1;
          tr = umax(tr, tau[prev * N + w]);
          prev = w;
        }
        tr = umax(tr, tau[prev * N + first]);
      }
      g.ring[msk] = tr;
    }
    u64 mt = 0;
    for (int i = lane; i < N * N; i += 32)
      if (i / N != i % N) mt = umax(mt, tau[i]);
    const u64 maxTau = warp_max(mt);
    u64 mog = 0;
    for (int l = lane; l < L; l += 32) mog = umax(mog, umax(g.O[l], g.G[l]));
    const u64 maxOG = warp_max(mog);
    // sum over layers of max over workers of (f + b), with overflow detection; the same for f and b
    // alone (saturated at 2^32) for the narrow path
    bool ovf = false;
    u64 part = 0, pf = 0, pb = 0;
    for (int l = lane; l < L; l += 32) {
      u64 m = 0, mf = 0, mb = 0;
      for (int w = 0; w < N; ++w) {
        const u64 a = fp[w * L + l], b = bp[w * L + l];
        if (a >= (1ull << 59) || b >= (1ull << 59)) ovf = true;  // then the bound fails anyway
        m = umax(m, a + b);
        mf = umax(mf, a);
        mb = umax(mb, b);
      }
      part = (part >= (1ull << 59) || m >= (1ull << 60)) ? (1ull << 59) : part + m;  // saturate
      pf = umin(pf + umin(mf, 1ull << 32), 1ull << 32);
      pb = umin(pb + umin(mb, 1ull << 32), 1ull << 32);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      pf = umin(pf + __shfl_xor_sync(0xffffffffu, pf, o), 1ull << 32);
      pb = umin(pb + __shfl_xor_sync(0xffffffffu, pb, o), 1ull << 32);
    }
    u64 sumMax = part;  // every lane's part <= 2^59 + 2^60, so the 32-lane sum cannot wrap
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sumMax += __shfl_xor_sync(0xffffffffu, sumMax, o);
    ovf = __any_sync(0xffffffffu, ovf) || sumMax >= (1ull << 59);
    if (lane == 0) {
      const u64 maxBytes = umax(maxOG, sumP);
      // bytes * tau + 999999 < 2^64
      const u64 hi = __umul64hi(maxBytes, maxTau), lo = maxBytes * maxTau;
      if (hi != 0 || lo + 999999ull < lo) ovf = true;
      const u64 maxX = ovf ? 0 : (lo + 999999ull) / 1000000ull;
      const u64 maxXog = (maxOG * maxTau + 999999ull) / 1000000ull;  // <= maxX
      // bound = sumMax + 16 + 28 maxX < 2^59 (N <= 8; 32 + 60 maxX for N <= 16, wide records; sumMax <
      // 2^59 and maxX < 2^55 here: no wrap). The host path (autopipe_set_state) uses the same rule.
      u64 bound = ~0ull, bound32 = ~0ull;
      if (maxX >= (1ull << 55)) ovf = true;
      const bool wideN = N > MAXN;
      if (!ovf) {
        bound = sumMax + (wideN ? 32 : 16) + (wideN ? 60 : 28) * maxX;
        bound32 = sumMax + (wideN ? 32 : 16) + (wideN ? 30 : 14) * maxXog;
      }
      if (bound >= (1ull << 59)) ovf = true;
      const u64 path32 = (!ovf && bound32 < 0xFFFFFFF0ull) ? 2ull : 0ull;
      const u64 lim = (1ull << 31) - 16;
      const u64 narrow = (!ovf && pf <= lim && pb <= lim && maxOG < (1ull << 31) && maxTau < (1ull << 32)) ? 4ull : 0ull;
      g.status[0] = (ovf ? 1ull : 0ull) | path32 | narrow;
      g.status[1] = bound;
    }
    return;
  }
  // link tables: one thread per (s, l), s in [0, N-2], l in [0, L-2]; then one per (l, u, v) for the
  // single-worker boundary table xp (forward and backward transfer of the cut after layer l)
  const int t = (blockIdx.x * blockDim.x + threadIdx.x) - (scan_warps + 1) * 32;
  const int per = (L > 1) ? L - 1 : 0;
  if (t < 0 || per == 0) return;
  if (t >= (N - 1) * per) {
    const int q = t - (N - 1) * per;
    if (q >= per * N * N) return;
    const int l = q / (N * N), u = (q / N) % N, v = q % N;
    u64 *x = g.xp + 2 * ((l * TAUW + u) * TAUW + v);
    x[0] = (u == v) ? 0ull : xfer(g.O[l], tau[u * N + v]);
    x[1] = (u == v) ? 0ull : xfer(g.G[l + 1], tau[v * N + u]);
    return;
  }
  const int s = t / per, l = t % per;
  const u64 cf = xfer(g.O[l], tau[s * N + s + 1]);
  const u64 cb = xfer(g.G[l + 1], tau[(s + 1) * N + s]);
  g.Z[s * L + l] = cf + cb;
  g.LM[s * L + l] = umax(cf, cb);
  g.Z32[s * L + l] = (u32)(cf + cb);
  g.LM32[s * L + l] = (u32)umax(cf, cb);
}

int launch_build_state(const DevTables &g, const u64 *fp, const u64 *bp, const u64 *P, const u64 *tau, u64 sumP,
                       cudaStream_t st) {
  const int scan_warps = 3 * (int)g.N + 1;
  const int per = (int)g.L > 1 ? (int)g.L - 1 : 0;
  const int links = ((int)g.N - 1) * per + per * (int)(g.N * g.N);
  const int threads = (scan_warps + 1) * 32 + (links > 0 ? links : 0);
  const int bs = 256;
  const int blocks = (threads + bs - 1) / bs;
  k_build_state<<<blocks, bs, 0, st>>>(g, fp, bp, P, tau, sumP, scan_warps);
  return 1;
}

}  // namespace ap
