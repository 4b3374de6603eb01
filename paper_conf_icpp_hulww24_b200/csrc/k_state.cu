// k_state.cu — rows a1 and a2: state ingest (per-worker prefix sums of f, b, f+b and of the weight
// bytes) and the r = 1 link tables, built on the device after every autopipe_set_state.
//
// Table 1 inputs: FP_ij, BP_ij (N x L ns), P_i (L bytes), O_i, G_i (L bytes) and
// the per-link inverse bandwidth (reading C-5). One launch, two roles:
//   warps 0 .. 3N   : one row each — warp-shuffle inclusive scan (__shfl_up_sync) over 32-element
//                     chunks with a running carry, written as an exclusive prefix of L + 1 entries
//                     (rows: PF[w], PB[w], PC[w] = prefix of f + b, and PP);
//   remaining warps : link tables Z[s][l] = cf + cb and LM[s][l] = max(cf, cb) for the boundary
//                     between worker s and s + 1 at a cut after layer l, with
//                     cf = ceil(O[l] * tau[s][s+1] / 1e6) and cb = ceil(G[l+1] * tau[s+1][s] / 1e6)
//                     (forward activation / backward input gradient, reading C-6).
// 32-bit copies of PC, Z, LM are written when the host selected the 32-bit search path.
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

// raw: fp [N][L], bp [N][L], P [L]
__global__ void k_build_state(DevTables g, const u64 *__restrict__ fp, const u64 *__restrict__ bp,
                              const u64 *__restrict__ P, int path32, int scan_warps) {
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
    } else if (kind == 1) {
      dst = g.PB + w * Lp1;
    } else {
      dst = g.PC + w * Lp1;
      if (path32) dst32 = g.PC32 + w * Lp1;
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
  // link tables: one thread per (s, l), s in [0, N-2], l in [0, L-2]
  const int t = (blockIdx.x * blockDim.x + threadIdx.x) - scan_warps * 32;
  const int per = (L > 1) ? L - 1 : 0;
  if (per == 0 || t >= (N - 1) * per) return;
  const int s = t / per, l = t % per;
  const u64 cf = xfer(g.O[l], g.tau[s * 8 + s + 1]);
  const u64 cb = xfer(g.G[l + 1], g.tau[(s + 1) * 8 + s]);
  g.Z[s * L + l] = cf + cb;
  g.LM[s * L + l] = umax(cf, cb);
  if (path32) {
    g.Z32[s * L + l] = (u32)(cf + cb);
    g.LM32[s * L + l] = (u32)umax(cf, cb);
  }
}

int launch_build_state(const DevTables &g, const u64 *fp, const u64 *bp, const u64 *P, int path32,
                       cudaStream_t st) {
  const int scan_warps = 3 * (int)g.N + 1;
  const int links = ((int)g.N - 1) * ((int)g.L > 1 ? (int)g.L - 1 : 0);
  const int threads = scan_warps * 32 + (links > 0 ? links : 0);
  const int bs = 256;
  const int blocks = (threads + bs - 1) / bs;
  k_build_state<<<blocks, bs, 0, st>>>(g, fp, bp, P, path32, scan_warps);
  return 1;
}

}  // namespace ap
