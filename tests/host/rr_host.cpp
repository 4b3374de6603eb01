// CPU test harness (tests/test_host_rr.py): the round-robin recurrence of the GPU path
// (paper_conf_icpp_hulww24_b200/csrc/rr.cuh, reading F-5) compiled for the host, scoring records
// of a state read from a text dump; the test compares each T with the oracle's
// (oracle/roundrobin.py), which the dump carries. argv: dump [cap] — with cap, every record stops
// the recurrence after `cap` rounds and takes the Bellman-Ford in the growth bounds' bracket (the
// path of the GPU's deferred and long-transient records).
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "rr.cuh"

using namespace ap;

int main(int argc, char **argv) {
  FILE *f = fopen(argv[1], "r");
  if (!f) return 2;
  unsigned L, N;
  if (fscanf(f, "%u %u", &L, &N) != 2) return 2;
  std::vector<u64> fp(N * L), bp(N * L), O(L), G(L), P(L), tau(N * N);
  for (auto *v : {&fp, &bp, &O, &G, &P, &tau})
    for (auto &x : *v)
      if (fscanf(f, "%llu", &x) != 1) return 2;
  const unsigned Lp1 = L + 1;
  std::vector<u64> PF(N * Lp1, 0), PB(N * Lp1, 0), PP(Lp1, 0), T16(TAUW * TAUW, 0);
  for (unsigned w = 0; w < N; ++w)
    for (unsigned l = 0; l < L; ++l) {
      PF[w * Lp1 + l + 1] = PF[w * Lp1 + l] + fp[w * L + l];
      PB[w * Lp1 + l + 1] = PB[w * Lp1 + l] + bp[w * L + l];
    }
  for (unsigned l = 0; l < L; ++l) PP[l + 1] = PP[l] + P[l];
  for (unsigned u = 0; u < N; ++u)
    for (unsigned v = 0; v < N; ++v) T16[u * TAUW + v] = u == v ? 0 : tau[u * N + v];
  // the single-worker boundary table of the state kernel (k_state.cu), for the closed form
  std::vector<u64> xp(2 * (size_t)(L > 1 ? L - 1 : 1) * TAUW * TAUW, 0);
  for (unsigned l = 0; l + 1 < L; ++l)
    for (unsigned u = 0; u < N; ++u)
      for (unsigned v = 0; v < N; ++v) {
        u64 *x = &xp[2 * ((l * TAUW + u) * TAUW + v)];
        x[0] = u == v ? 0 : xfer(O[l], tau[u * N + v]);
        x[1] = u == v ? 0 : xfer(G[l + 1], tau[v * N + u]);
      }
  std::vector<DivEnt> dt(MAXNW + 1);
  for (unsigned i = 0; i <= (unsigned)MAXNW; ++i) {
    const unsigned dd = i ? i : 1;
    const DivR<16> d(dd);
    u32 m32, k32;
    Div32::make(dd, m32, k32);
    dt[i] = DivEnt{d.m, d.sh, d.Ms, m32, k32, 0u, 0u};
  }
  SmemTab t;
  t.PF = PF.data(); t.PB = PB.data(); t.PP = PP.data(); t.O = O.data(); t.G = G.data(); t.tau = T16.data();
  t.ring = nullptr; t.PF32 = t.PB32 = t.tau32 = t.PC32 = nullptr; t.dv = dt.data(); t.xp = xp.data();
  t.L = (int)L; t.Lp1 = (int)Lp1;
  const int cap = argc > 2 ? atoi(argv[2]) : 0;
  int M, sync;
  if (fscanf(f, "%d %d", &M, &sync) != 2) return 2;
  int bad = 0, n = 0;
  for (int i = 0; i < M; ++i) {
    u64 lo, hi, ref;
    if (fscanf(f, "%llx %llx %llu", &lo, &hi, &ref) != 3) return 2;
    int S;
    P8 p;
    u64 T = U64MAX;
    if (decode_record(lo, hi, (int)L, (int)N, S, p)) {
      if (cap > 0) {
        RRSetup R;
        rr_setup(t, S, p, sync, R);
        if (S == 1) {
          T = umax(rr_single_stage(R), R.Tsync);
        } else {
          u64 a, b;
          const bool met = rr_sim(R, (u32)cap, U64MAX, a, b, nullptr) == RR_MET;
          T = umax(met ? a : rr_ceil_bf(R, a, b), R.Tsync);
        }
      } else {
        T = rr_time(t, S, p, sync);
      }
    }
    ++n;
    if (T != ref) {
      ++bad;
      if (bad < 10) printf("record %d: got %llu, oracle %llu\n", i, T, ref);
    }
  }
  printf("scored %d bad %d\n", n, bad);
  return bad ? 1 : 0;
}
