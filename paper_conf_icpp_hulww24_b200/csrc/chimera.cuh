// chimera.cuh — NEXT row f3: Chimera's bidirectional pipelines (reading F-6; oracle/chimera.py).
//
// "Chimera effectively maps stages of the model in linear and opposite orders across two pipelines"
// (AutoPipe applied to it in Fig. 13). A Chimera partition has
// one worker per stage: stage s runs on w_s in the "down" pipeline and on w_{S-1-s} in the "up" one,
// so every worker g holds down stage g and up stage S-1-g. An iteration's M micro-batches split
// ceil(M/2) down and floor(M/2) up; each pipeline keeps DAPPLE's per-stage order (1F1B with flush);
// a worker interleaves its two lists by readiness: repeatedly the op with the earliest start
// max(worker free, input ready) among the list heads whose input exists runs next (ties: lower
// worker, then down). Transfers start when their producing op ends, FIFO per directed link (the two
// pipelines share the links between neighbouring workers); stage s's two copies synchronise after
// both last backwards. T = max_s (later last backward of the copies + sync).
//
// One thread per partition runs that list schedule directly: per worker its free time and two list
// positions, per pipeline and boundary a ring of the last transfer completions (a boundary never has
// more than S <= 8 outstanding: a stage runs ahead of its successor by at most its warm-up), per
// directed neighbour link its free time. Each step picks the earliest start among the 2S list heads,
// whose start times are cached and recomputed only where the step changed them.
#pragma once
#include "eval.cuh"

namespace ap {

// ring of transfer completions per pipeline and boundary: a stage runs ahead of its successor by at
// most its warm-up (<= S), so 8 slots serve 16-byte records and 16 the wide ones
template <typename P>
struct ChRing {
  static constexpr int N = P::MS;
};

// op at position i of DAPPLE's list for stage s of an S-stage pipeline with M micro-batches:
// kind (0 = F, 1 = B) and micro-batch
__device__ __forceinline__ void dapple_op(int S, int s, u32 M, u32 i, int &kind, u32 &k) {
  const u32 n = (u32)(S - s) < M ? (u32)(S - s) : M;
  if (i < n) {
    kind = 0;
    k = i;
    return;
  }
  const u32 q = i - n;
  if (q < 2 * (M - n)) {
    kind = (int)(q & 1u) ^ 1;  // even q: B(q/2), odd q: F(q/2 + n)
    k = (q >> 1) + ((q & 1u) ? n : 0u);
  } else {
    kind = 1;
    k = i - M;
  }
}

// T_ns of a validated partition (16-byte P8 or wide P16) under Chimera; UINT64_MAX if a stage is
// replicated.
template <typename P>
static __device__ __noinline__ u64 chimera_time(const SmemTab &t, int S, const P &p, const ModelP &m) {
  constexpr int MS = P::MS, CH_RING = ChRing<P>::N;
  int wk[MS];
  for (int s = 0; s < S; ++s) {
    const u32 mask = p.mask(s);
    if (__popc(mask) != 1) return U64MAX;
    wk[s] = __ffs(mask) - 1;
  }
  const u32 Mp[2] = {(m.M + 1) / 2, m.M / 2};
  // durations: group g (worker wk[g]) runs down stage g and up stage S-1-g
  u64 dur[MS][2][2];  // [g][pipe][kind]
  for (int g = 0; g < S; ++g) {
    const int w = wk[g];
    for (int pipe = 0; pipe < 2; ++pipe) {
      const int s = pipe == 0 ? g : S - 1 - g;
      const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
      const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
      dur[g][pipe][0] = t.PF[w * t.Lp1 + e + 1] - t.PF[w * t.Lp1 + a];
      dur[g][pipe][1] = t.PB[w * t.Lp1 + e + 1] - t.PB[w * t.Lp1 + a];
    }
  }
  // neighbour links: right[g] = w_g -> w_{g+1} (down forward g, up backward), left[g] = w_{g+1} -> w_g
  u64 lright[MS], lleft[MS], xr_dn[MS], xl_dn[MS], xl_up[MS], xr_up[MS];
  for (int g = 0; g + 1 < S; ++g) {
    lright[g] = lleft[g] = 0;
    const u64 tr = t.tau[wk[g] * TAUW + wk[g + 1]], tl = t.tau[wk[g + 1] * TAUW + wk[g]];
    const int e = p.cut(g);          // down boundary g: after stage g
    const int eu = p.cut(S - 2 - g);  // up boundary u = S-2-g: after up stage u (the same layers as stage u)
    xr_dn[g] = xfer(t.O[e], tr);       // down forward g on the right link
    xl_dn[g] = xfer(t.G[e + 1], tl);   // down backward g on the left link
    xl_up[g] = xfer(t.O[eu], tl);      // up forward u: worker of up stage u (w_{g+1}) -> w_g
    xr_up[g] = xfer(t.G[eu + 1], tr);  // up backward u: w_g -> w_{g+1}
  }
  // boundary rings: [pipe][boundary][slot], forward and backward, with produced counts
  u64 fr[2][MS - 1][CH_RING], br[2][MS - 1][CH_RING];
  u32 fcnt[2][MS - 1], bcnt[2][MS - 1];
  u64 fre[MS], lastb[MS][2];
  u32 pos[MS][2];
  for (int g = 0; g < S; ++g) {
    fre[g] = 0;
    pos[g][0] = pos[g][1] = 0;
    lastb[g][0] = lastb[g][1] = 0;
  }
  for (int q = 0; q < S - 1; ++q) fcnt[0][q] = fcnt[1][q] = bcnt[0][q] = bcnt[1][q] = 0;
  // the start time of every list head (UINT64_MAX: exhausted or its input not produced yet), kept
  // up to date incrementally: an op changes only its worker's two heads and the head that consumes
  // the transfer it starts, so a step recomputes at most four heads and then picks the earliest
  // start among the 2S cached ones (scan order = the tie order: lower worker, then down)
  auto head_start = [&](int g, int pipe) -> u64 {
    const u32 M = Mp[pipe];
    if (pos[g][pipe] >= 2 * M) return U64MAX;
    const int s = pipe == 0 ? g : S - 1 - g;  // stage index within the pipeline
    int kind;
    u32 k;
    dapple_op(S, s, M, pos[g][pipe], kind, k);
    u64 ready = 0;
    if (kind == 0 && s > 0) {
      if (k >= fcnt[pipe][s - 1]) return U64MAX;
      ready = fr[pipe][s - 1][k & (CH_RING - 1)];
    } else if (kind == 1 && s < S - 1) {
      if (k >= bcnt[pipe][s]) return U64MAX;
      ready = br[pipe][s][k & (CH_RING - 1)];
    }
    return umax(fre[g], ready);
  };
  // the cached head starts stay in registers: the scan and the updates index them only with
  // unrolled (compile-time) indices, updates by selects (the head recomputations read the other
  // arrays once per step)
  u64 hs[MS][2];
#pragma unroll
  for (int g = 0; g < MS; ++g) {
    hs[g][0] = g < S ? head_start(g, 0) : U64MAX;
    hs[g][1] = g < S ? head_start(g, 1) : U64MAX;
  }
  const u32 total = 2u * (u32)S * m.M;
  for (u32 step = 0; step < total; ++step) {
    u64 best = U64MAX;
    int bg = -1, bp = 0;
#pragma unroll
    for (int g = 0; g < MS; ++g)
#pragma unroll
      for (int pipe = 0; pipe < 2; ++pipe)
        if (hs[g][pipe] < best) {
          best = hs[g][pipe];
          bg = g;
          bp = pipe;
        }
    if (bg < 0) return U64MAX;  // cannot happen: the lists of both pipelines are live
    const int s = bp == 0 ? bg : S - 1 - bg;
    int bkind;
    u32 bk;
    dapple_op(S, s, Mp[bp], pos[bg][bp], bkind, bk);
    const u64 end = best + dur[bg][bp][bkind];
    fre[bg] = end;
    ++pos[bg][bp];
    int cg = -1;  // the group whose head consumes the transfer this op starts
    if (bkind == 0 && s < S - 1) {
      // forward transfer to the pipeline's next stage: down g -> g+1 on the right link, up on the left
      u64 fin;
      if (bp == 0) {
        fin = umax(end, lright[bg]) + xr_dn[bg];
        lright[bg] = fin;
        cg = bg + 1;
      } else {
        fin = umax(end, lleft[bg - 1]) + xl_up[bg - 1];
        lleft[bg - 1] = fin;
        cg = bg - 1;
      }
      fr[bp][s][bk & (CH_RING - 1)] = fin;
      ++fcnt[bp][s];
    }
    if (bkind == 1) {
      lastb[bg][bp] = end;
      if (s > 0) {  // backward transfer to the pipeline's previous stage
        u64 fin;
        if (bp == 0) {
          fin = umax(end, lleft[bg - 1]) + xl_dn[bg - 1];
          lleft[bg - 1] = fin;
          cg = bg - 1;
        } else {
          fin = umax(end, lright[bg]) + xr_up[bg];
          lright[bg] = fin;
          cg = bg + 1;
        }
        br[bp][s - 1][bk & (CH_RING - 1)] = fin;
        ++bcnt[bp][s - 1];
      }
    }
    const u64 h0 = head_start(bg, 0), h1 = head_start(bg, 1), hc = cg >= 0 ? head_start(cg, bp) : 0;
#pragma unroll
    for (int g = 0; g < MS; ++g) {
      if (g == bg) hs[g][0] = h0, hs[g][1] = h1;
      if (g == cg) {
        if (bp == 0) hs[g][0] = hc;
        else hs[g][1] = hc;
      }
    }
  }
  u64 T = 0;
  for (int s = 0; s < S; ++s) {
    // stage s: down copy on group s, up copy on group S-1-s
    u64 fin = umax(lastb[s][0], lastb[S - 1 - s][1]);
    if (wk[s] != wk[S - 1 - s]) {
      const int a = (s == 0) ? 0 : p.cut(s - 1) + 1;
      const int e = (s == S - 1) ? t.L - 1 : p.cut(s);
      fin += sync_time<P::MN>((int)m.sync, t.PP[e + 1] - t.PP[a], (1u << wk[s]) | (1u << wk[S - 1 - s]), t.tau, t.dv);
    }
    T = umax(T, fin);
  }
  return T;
}

}  // namespace ap
