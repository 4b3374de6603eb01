// autopipe.cu — host side of the C-ABI (include/autopipe.h): argument validation, the overflow
// rules of SPEC.md §7, the integer-path choice, device buffers, shard/index arithmetic of the search
// space (SPEC.md §5) and kernel launches. No score is ever computed here: every T_ns comes from the
// sm_100a kernels in k_state.cu / k_eval.cu / k_search.cu / k_search_r1.cu.
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>

#include "../../include/autopipe.h"
#include "internal.h"

using namespace ap;

typedef unsigned __int128 u128;

static const u64 LIMIT_BYTES = 1ull << 56;   // any single byte count (and sum P)
static const u64 LIMIT_TIME = 1ull << 59;    // the largest modelled sum (SPEC.md §7)
static const u64 LIMIT_TIME32 = 0xFFFFFFF0u; // 32-bit search path
static const int MAX_BLOCKS = 148 * 32;

struct autopipe_ctx {
  int device = 0, sms = 148;
  char err[512] = {0};
  bool has_profile = false, has_state = false;
  bool state_on_device = false;  // last state came from device pointers: status not yet read
  u32 L = 0, N = 0;
  int path32 = 0;
  // narrow eval path (status bit 2): every per-worker stage sum of f or of b < 2^31 - 16, activation
  // and gradient bytes < 2^31 and tau < 2^32, so stage costs and shard overlaps are 32-bit
  int narrow = 0;
  u64 launches = 0;
  u64 maxOG = 0, sumP = 0;
  u64 bound = 0;  // the state's bound on modelled sums (SPEC.md §7)
  ModelP model{SCHED_PIPEDREAM, SYNC_RING, 1, 0};  // row f3: schedule variant + sync scheme
  DevTables tab{};
  // device buffers
  u64 *d_raw = nullptr;      // fp [N*L] | bp [N*L] | tau [N*N] (contiguous, one copy) ... | P [255] at RAW_P
  u64 *d_tables = nullptr;   // all DevTables arrays
  BlockOut *d_blocks = nullptr;
  ResultDev *d_result = nullptr;
  void *d_work = nullptr;
  void *d_nslots = nullptr;  // neighbourhood slots (records), times, count
  u64 *d_ntimes = nullptr, *d_ncount = nullptr, *h_ncount = nullptr;
  // chunk counters of the eval kernel's dynamic schedule: one slot per launch, round-robin, so
  // launches on different streams never share one
  static const int NCTR = 256;
  u32 *d_ctr = nullptr;
  // row f4, round-robin replicas: the deferral queue of the eval kernels (RRQueue) and the event of
  // the last drain that used it (the next evaluation's stream waits for it)
  static const u32 RRQ_CAP = 1u << 14;
  u64 *d_rrq = nullptr;
  u32 *d_rrq_n = nullptr;
  cudaEvent_t ev_rrq = nullptr;
  u32 ctr_next = 0;
  // the same for the search kernels' schedules (SEARCH_SCHED_BYTES per launch)
  unsigned char *d_sched = nullptr;
  u32 sched_next = 0;
  void *h_work = nullptr;  // pinned mirror of d_work (r = 1 schedules)
  size_t work_bytes = 0;
  // pinned host staging
  u64 *h_stage = nullptr;    // fp | bp | tau (pinned staging of set_state, the layout of d_raw)
  u64 *h_prof = nullptr;     // O [255] | G [255] | P [255] (pinned staging of load_profile)
  // load_profile copies on its own stream (no host wait); set_state's stream waits for ev_prof.
  // ev_stage / ev_prof mark the last copies out of the two staging buffers (a refill waits for them).
  cudaStream_t pstream = nullptr;
  cudaEvent_t ev_prof = nullptr, ev_stage = nullptr;
  bool prof_pending = false, stage_pending = false;
  ResultDev *h_result = nullptr;
  u64 *h_status = nullptr;   // pinned copy of the device status word
  u64 binom[BINOM_N][BINOM_K];
  // the search's kernels (one or two per S) run on NAUX internal streams, forked from and joined back
  // into the caller's stream: a short model's space is a dozen small launches, latency-bound in series
  static const int NAUX = 4;
  cudaStream_t aux[NAUX] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t ev_fork = nullptr, ev_join[NAUX] = {nullptr, nullptr, nullptr, nullptr};
  // optional device timing of the search kernels (autopipe_set_timing)
  bool timing = false;
  u32 search_options = 0;  // autopipe_set_search_options
  // a ring of event pairs: search k (counted while timing is on) records pair k % TRING, so the
  // times of asynchronous searches can be read after the fact (autopipe_search_times)
  static const int TRING = 64;
  cudaEvent_t ev0[TRING] = {}, ev1[TRING] = {};
  u64 tcount = 0, tread = 0;  // timed searches recorded / already returned by autopipe_search_times
  // recorded after a search's schedule copies: the pinned schedule slots are rewritten only after it
  // (an asynchronous search returns before its copies have run)
  cudaEvent_t ev_hwork = nullptr;
  bool hwork_pending = false;
  // row e, cross-shard bound: the device word later searches' r = 1 sweeps start from
  // (autopipe_set_search_bound), and the seed-only call's own schedule slots (upper half of the work
  // areas) with their own copy event
  // The bound is valid only for the state, schedule and space it was seeded on: `gen` counts profile,
  // state and schedule changes; a seed call records (gen, s_min, s_max, flags), set_search_bound
  // copies that key, and a search applies the bound only when its own key matches.
  const u64 *d_bound = nullptr;
  u64 gen = 0, seed_gen = ~0ull, bound_gen = ~0ull;
  u32 seed_key[3] = {0, 0, 0}, bound_key[3] = {0, 0, 0};
  cudaEvent_t ev_hseed = nullptr;
  bool hseed_pending = false;
};

static char g_create_err[256] = "";
// word offset of P in d_raw: after the largest fp | bp | tau block (2 * 16 * 255 + 16 * 16 words)
static const size_t RAW_P = 2 * (size_t)MAXNW * MAXL + (size_t)TAUW * TAUW;

// The round-robin deferral queue for an evaluation on stream st (row f4): st first waits for the
// previous drain that used the queue, and the caller records ev_rrq after its own launch.
static RRQueue rr_queue(autopipe_ctx *c, cudaStream_t st, bool wide) {
  RRQueue q;
  if (c->model.sched != SCHED_RR || wide || (c->search_options & AUTOPIPE_RR_NO_DEFER)) return q;
  cudaStreamWaitEvent(st, c->ev_rrq, 0);
  q.buf = c->d_rrq;
  q.n = c->d_rrq_n;
  q.cap = autopipe_ctx::RRQ_CAP;
  q.rounds = (c->search_options & AUTOPIPE_RR_DEFER_ALL) ? 1u : RR_DEFER_ROUNDS;
  return q;
}
static void rr_queue_done(autopipe_ctx *c, cudaStream_t st, const RRQueue &q) {
  if (q.buf) cudaEventRecord(c->ev_rrq, st);
}

static u32 *next_counter(autopipe_ctx *c) { return c->d_ctr + (c->ctr_next++ % autopipe_ctx::NCTR); }
static void *next_sched(autopipe_ctx *c) {
  return c->d_sched + (size_t)SEARCH_SCHED_BYTES * (c->sched_next++ % autopipe_ctx::NCTR);
}

const char *ap::experiment_knob(const char *name) {
  static const bool on = [] {
    const char *v = getenv("AUTOPIPE_EXPERIMENTS");
    return v && v[0] == '1';
  }();
  if (!on) return nullptr;
  const char *v = getenv(name);
  return (v && *v) ? v : nullptr;
}

static int fail(autopipe_ctx *c, int code, const char *fmt, ...) {
  va_list ap_;
  va_start(ap_, fmt);
  vsnprintf(c->err, sizeof(c->err), fmt, ap_);
  va_end(ap_);
  return code;
}

static int cuda_fail(autopipe_ctx *c, cudaError_t e, const char *what) {
  return fail(c, AUTOPIPE_E_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

// RAII device switch: the caller's current device is restored on return.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

// C(n, k), n < 256, k <= 16, saturated at UINT64_MAX (only spaces below 2^64 are ever indexed)
static void host_binomials(u64 (*b)[BINOM_K]) {
  for (int n = 0; n < BINOM_N; ++n)
    for (int k = 0; k < BINOM_K; ++k) {
      if (k == 0) b[n][k] = 1;
      else if (n == 0) b[n][k] = 0;
      else {
        const u64 x = b[n - 1][k - 1], y = b[n - 1][k];
        b[n][k] = (x > U64MAX - y) ? U64MAX : x + y;
      }
    }
}

extern "C" int autopipe_create(int cuda_device, autopipe_ctx **out) {
  if (!out) {
    snprintf(g_create_err, sizeof(g_create_err), "out is NULL");
    return AUTOPIPE_E_INVAL;
  }
  *out = nullptr;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || cuda_device < 0 || cuda_device >= ndev) {
    snprintf(g_create_err, sizeof(g_create_err), "no CUDA device %d (%s)", cuda_device,
             e != cudaSuccess ? cudaGetErrorString(e) : "out of range");
    return AUTOPIPE_E_CUDA;
  }
  autopipe_ctx *c = new (std::nothrow) autopipe_ctx();
  if (!c) return AUTOPIPE_E_NOMEM;
  c->device = cuda_device;
  DeviceGuard dg(cuda_device);
  cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, cuda_device);
  host_binomials(c->binom);
  upload_binomials(c->binom);
  // device tables, sized for the limits (L = 255, N = 8): a few hundred KB
  const size_t Lp1 = MAXL + 1, NL = (size_t)MAXNW * Lp1, TT = (size_t)TAUW * TAUW;
  const size_t words = 3 * NL + Lp1 + 2 * MAXL + TT + 2 * 7 * MAXL + 2 + 256 + (size_t)MAXL * TT * 2;
  const size_t words32 = 3 * NL + 2 * 7 * MAXL;
  e = cudaMalloc(&c->d_tables, words * 8 + words32 * 4 + 64);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_raw, (2 * MAXNW * MAXL + MAXL + TT) * 8);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_blocks, sizeof(BlockOut) * MAX_BLOCKS);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_result, sizeof(ResultDev));
  c->work_bytes = 1 << 20;
  if (e == cudaSuccess) e = cudaMalloc(&c->d_work, c->work_bytes);
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_work, c->work_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_nslots, (size_t)NEIGH_ITEMS * NEIGH_MAXOPT * 16);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_ntimes, (size_t)NEIGH_ITEMS * NEIGH_MAXOPT * 8);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_ncount, 8);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_ctr, sizeof(u32) * autopipe_ctx::NCTR);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_rrq, sizeof(u64) * 3 * autopipe_ctx::RRQ_CAP);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_rrq_n, sizeof(u32));
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_rrq, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaMalloc(&c->d_sched, (size_t)SEARCH_SCHED_BYTES * autopipe_ctx::NCTR);
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_ncount, 8);
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_stage, (2 * MAXNW * MAXL + TT) * 8);
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_prof, 3 * MAXL * 8);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->pstream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_prof, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_stage, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_result, sizeof(ResultDev));
  if (e == cudaSuccess) e = cudaMallocHost(&c->h_status, 2 * sizeof(u64));
  if (e != cudaSuccess) {
    snprintf(g_create_err, sizeof(g_create_err), "allocation: %s", cudaGetErrorString(e));
    autopipe_destroy(c);
    return AUTOPIPE_E_NOMEM;
  }
  u64 *p = c->d_tables;
  c->tab.PF = p; p += NL;
  c->tab.PB = p; p += NL;
  c->tab.PC = p; p += NL;
  c->tab.PP = p; p += Lp1;
  c->tab.O = p; p += MAXL;
  c->tab.G = p; p += MAXL;
  c->tab.tau = p; p += TT;
  c->tab.Z = p; p += 7 * MAXL;
  c->tab.LM = p; p += 7 * MAXL;
  c->tab.status = p; p += 2;
  c->tab.ring = p; p += 256;
  c->tab.xp = p; p += (size_t)MAXL * TT * 2;
  u32 *q = (u32 *)p;
  c->tab.PC32 = q; q += NL;
  c->tab.PF32 = q; q += NL;
  c->tab.PB32 = q; q += NL;
  c->tab.Z32 = q; q += 7 * MAXL;
  c->tab.LM32 = q; q += 7 * MAXL;
  e = cudaMemset(c->d_tables, 0, words * 8 + words32 * 4 + 64);
  if (e != cudaSuccess) {
    snprintf(g_create_err, sizeof(g_create_err), "memset: %s", cudaGetErrorString(e));
    autopipe_destroy(c);
    return AUTOPIPE_E_CUDA;
  }
  *out = c;
  return AUTOPIPE_OK;
}

extern "C" void autopipe_destroy(autopipe_ctx *c) {
  if (!c) return;
  {
    DeviceGuard dg(c->device);
    cudaDeviceSynchronize();
    if (c->d_tables) cudaFree(c->d_tables);
    if (c->d_raw) cudaFree(c->d_raw);
    if (c->d_blocks) cudaFree(c->d_blocks);
    if (c->d_result) cudaFree(c->d_result);
    if (c->d_work) cudaFree(c->d_work);
    if (c->h_work) cudaFreeHost(c->h_work);
    if (c->d_nslots) cudaFree(c->d_nslots);
    if (c->d_ntimes) cudaFree(c->d_ntimes);
    if (c->d_ncount) cudaFree(c->d_ncount);
    if (c->d_ctr) cudaFree(c->d_ctr);
    if (c->d_rrq) cudaFree(c->d_rrq);
    if (c->d_rrq_n) cudaFree(c->d_rrq_n);
    if (c->ev_rrq) cudaEventDestroy(c->ev_rrq);
    if (c->d_sched) cudaFree(c->d_sched);
    if (c->h_ncount) cudaFreeHost(c->h_ncount);
    if (c->h_stage) cudaFreeHost(c->h_stage);
    if (c->h_prof) cudaFreeHost(c->h_prof);
    if (c->pstream) cudaStreamDestroy(c->pstream);
    if (c->ev_prof) cudaEventDestroy(c->ev_prof);
    if (c->ev_stage) cudaEventDestroy(c->ev_stage);
    if (c->h_result) cudaFreeHost(c->h_result);
    if (c->h_status) cudaFreeHost(c->h_status);
    if (c->ev_hwork) cudaEventDestroy(c->ev_hwork);
    if (c->ev_hseed) cudaEventDestroy(c->ev_hseed);
    for (int i = 0; i < autopipe_ctx::TRING; ++i) {
      if (c->ev0[i]) cudaEventDestroy(c->ev0[i]);
      if (c->ev1[i]) cudaEventDestroy(c->ev1[i]);
    }
    for (int i = 0; i < autopipe_ctx::NAUX; ++i) {
      if (c->aux[i]) cudaStreamDestroy(c->aux[i]);
      if (c->ev_join[i]) cudaEventDestroy(c->ev_join[i]);
    }
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  }
  delete c;
}

extern "C" const char *autopipe_last_error(const autopipe_ctx *c) { return c ? c->err : g_create_err; }

extern "C" int autopipe_load_profile(autopipe_ctx *c, uint32_t L, const uint64_t *O, const uint64_t *G,
                                     const uint64_t *P) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (L < 1 || L > MAXL) return fail(c, AUTOPIPE_E_INVAL, "L = %u outside [1, 255]", L);
  if (!O || !G || !P) return fail(c, AUTOPIPE_E_INVAL, "NULL profile array");
  u64 maxOG = 0;
  u128 sumP = 0;
  for (u32 l = 0; l < L; ++l) {
    if (O[l] >= LIMIT_BYTES || G[l] >= LIMIT_BYTES || P[l] >= LIMIT_BYTES)
      return fail(c, AUTOPIPE_E_OVERFLOW, "layer %u: a byte count >= 2^56", l);
    maxOG = umax(maxOG, umax((u64)O[l], (u64)G[l]));
    sumP += P[l];
  }
  if (sumP >= LIMIT_BYTES) return fail(c, AUTOPIPE_E_OVERFLOW, "sum of weight bytes >= 2^56");
  DeviceGuard dg(c->device);
  // O, G go straight to their (adjacent) tables, P to the raw area (the state kernel builds its
  // prefix): staged in pinned memory and copied on the context's profile stream without a host wait;
  // the next set_state's stream waits for the copies (ev_prof)
  cudaError_t e = cudaSuccess;
  if (c->prof_pending) e = cudaEventSynchronize(c->ev_prof);  // the staging buffer may still be read
  if (e != cudaSuccess) return cuda_fail(c, e, "load_profile sync");
  u64 *hO = c->h_prof, *hG = hO + MAXL, *hP = hG + MAXL;
  memcpy(hO, O, L * 8);
  memcpy(hG, G, L * 8);
  memcpy(hP, P, L * 8);
  e = cudaMemcpyAsync(c->tab.O, hO, (MAXL + L) * 8, cudaMemcpyHostToDevice, c->pstream);
  if (e == cudaSuccess) e = cudaMemcpyAsync(c->d_raw + RAW_P, hP, L * 8, cudaMemcpyHostToDevice, c->pstream);
  if (e == cudaSuccess) e = cudaEventRecord(c->ev_prof, c->pstream);
  if (e != cudaSuccess) return cuda_fail(c, e, "load_profile copy");
  c->prof_pending = true;
  c->L = L;
  c->maxOG = maxOG;
  c->sumP = (u64)sumP;
  c->has_profile = true;
  c->has_state = false;
  c->path32 = 0;
  ++c->gen;
  return AUTOPIPE_OK;
}

extern "C" int autopipe_set_state(autopipe_ctx *c, uint32_t N, const uint64_t *fp, const uint64_t *bp,
                                  const uint64_t *tau, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!c->has_profile) return fail(c, AUTOPIPE_E_STATE, "set_state before load_profile");
  if (N < 1 || N > MAXNW) return fail(c, AUTOPIPE_E_INVAL, "N = %u outside [1, 16]", N);
  if (!fp || !bp || !tau) return fail(c, AUTOPIPE_E_INVAL, "NULL state array");
  const u32 L = c->L;
  // overflow rules (SPEC.md §7)
  u64 maxTau = 0;
  for (u32 u = 0; u < N; ++u)
    for (u32 v = 0; v < N; ++v)
      if (u != v) maxTau = umax(maxTau, (u64)tau[u * N + v]);
  const u64 maxBytes = umax(c->maxOG, c->sumP);
  if ((u128)maxBytes * maxTau + 999999u >= ((u128)1 << 64))
    return fail(c, AUTOPIPE_E_OVERFLOW, "bytes * tau reaches 2^64");
  const u64 maxX = (u64)(((u128)maxBytes * maxTau + 999999u) / 1000000u);
  const u64 maxXog = (u64)(((u128)c->maxOG * maxTau + 999999u) / 1000000u);
  u128 sumMax = 0;
  for (u32 l = 0; l < L; ++l) {
    u128 m = 0;
    for (u32 w = 0; w < N; ++w) {
      const u128 v = (u128)fp[w * L + l] + bp[w * L + l];
      if (v > m) m = v;
    }
    sumMax += m;
  }
  // up to 7 boundaries (N <= 8) or 15 (N <= 16, wide records): 4 transfer bounds per boundary, one
  // rounding per stage (SPEC.md §7)
  const bool wideN = N > (u32)MAXN;
  const u128 bound = sumMax + (wideN ? 32 : 16) + (u128)(wideN ? 60 : 28) * maxX;
  if (bound >= LIMIT_TIME) return fail(c, AUTOPIPE_E_OVERFLOW, "modelled times reach 2^59 ns");
  const u128 bound32 = sumMax + (wideN ? 32 : 16) + (u128)(wideN ? 30 : 14) * maxXog;
  c->path32 = bound32 < LIMIT_TIME32 ? 1 : 0;
  {
    u128 sf = 0, sb = 0;
    for (u32 l = 0; l < L; ++l) {
      u64 mf = 0, mb = 0;
      for (u32 w = 0; w < N; ++w) {
        mf = umax(mf, (u64)fp[w * L + l]);
        mb = umax(mb, (u64)bp[w * L + l]);
      }
      sf += mf;
      sb += mb;
    }
    const u128 lim = ((u128)1 << 31) - 16;
    c->narrow = (sf <= lim && sb <= lim && c->maxOG < (1ull << 31) && maxTau < (1ull << 32)) ? 1 : 0;
  }
  c->bound = (u64)bound;
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  // stage into pinned memory (fp | bp | tau contiguous: one truly asynchronous copy); a refill waits
  // only for the previous copy out of the buffer (ev_stage), not for the stream's other work
  cudaError_t e = cudaSuccess;
  if (c->stage_pending) e = cudaEventSynchronize(c->ev_stage);
  if (e != cudaSuccess) return cuda_fail(c, e, "set_state sync");
  const size_t NL = (size_t)N * L;
  u64 *hf = c->h_stage, *hb = hf + NL, *ht = hb + NL;
  memcpy(hf, fp, NL * 8);
  memcpy(hb, bp, NL * 8);
  memcpy(ht, tau, (size_t)N * N * 8);
  u64 *rf = c->d_raw, *rb = rf + NL, *rt = rb + NL, *rP = c->d_raw + RAW_P;
  e = cudaStreamWaitEvent(st, c->ev_prof, 0);  // the profile's copies
  if (e == cudaSuccess) e = cudaMemcpyAsync(rf, hf, (2 * NL + (size_t)N * N) * 8, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaEventRecord(c->ev_stage, st);
  if (e != cudaSuccess) return cuda_fail(c, e, "set_state copy");
  c->stage_pending = true;
  c->tab.L = L;
  c->tab.N = N;
  c->tab.Lp1 = L + 1;
  c->N = N;
  c->launches += launch_build_state(c->tab, rf, rb, rP, rt, c->sumP, st);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "state kernel launch");
  c->has_state = true;
  c->state_on_device = false;
  ++c->gen;
  return AUTOPIPE_OK;
}

extern "C" int autopipe_set_state_device(autopipe_ctx *c, uint32_t N, const uint64_t *d_fp, const uint64_t *d_bp,
                                         const uint64_t *d_tau, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!c->has_profile) return fail(c, AUTOPIPE_E_STATE, "set_state before load_profile");
  if (N < 1 || N > MAXNW) return fail(c, AUTOPIPE_E_INVAL, "N = %u outside [1, 16]", N);
  if (!d_fp || !d_bp || !d_tau) return fail(c, AUTOPIPE_E_INVAL, "NULL state array");
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  c->tab.L = c->L;
  c->tab.N = N;
  c->tab.Lp1 = c->L + 1;
  c->N = N;
  const u64 *rP = c->d_raw + RAW_P;
  cudaError_t ew = cudaStreamWaitEvent(st, c->ev_prof, 0);  // the profile's copies
  if (ew != cudaSuccess) return cuda_fail(c, ew, "set_state_device wait");
  c->launches += launch_build_state(c->tab, (const u64 *)d_fp, (const u64 *)d_bp, rP, (const u64 *)d_tau, c->sumP, st);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "state kernel launch");
  c->has_state = true;
  c->state_on_device = true;  // overflow / path status is read from the device when first needed
  ++c->gen;
  return AUTOPIPE_OK;
}

// For a state given in device memory: fetch the status the state kernel computed (synchronises
// `stream`). Returns AUTOPIPE_E_OVERFLOW if the state violates SPEC.md §7.
static int sync_status(autopipe_ctx *c, cudaStream_t st) {
  if (!c->state_on_device) return AUTOPIPE_OK;
  cudaError_t e = cudaMemcpyAsync(c->h_status, c->tab.status, 2 * sizeof(u64), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(c, e, "state status");
  c->state_on_device = false;
  c->path32 = (c->h_status[0] & 2) ? 1 : 0;
  c->narrow = (c->h_status[0] & 4) ? 1 : 0;
  c->bound = c->h_status[1];
  if (c->h_status[0] & 1) {
    c->has_state = false;
    return fail(c, AUTOPIPE_E_OVERFLOW, "device state: bytes * tau reaches 2^64 or modelled times reach 2^59 ns");
  }
  return AUTOPIPE_OK;
}

// Row f3: a schedule other than PipeDream scales sums by up to 16 (M + 1) (an iteration of M
// micro-batches, recomputation, every op and transfer on a critical path); refuse states for which
// that could reach 2^63. Reads the device status first for a state set from device memory.
static int check_model(autopipe_ctx *c, cudaStream_t st, bool wide = false) {
  if (c->model.sched == SCHED_PIPEDREAM) return AUTOPIPE_OK;
  if (c->model.sched == SCHED_RR && wide)
    return fail(c, AUTOPIPE_E_INVAL, "round-robin replicas use 16-byte records (no wide calls)");
  int rc = sync_status(c, st);
  if (rc) return rc;
  if (c->model.sched == SCHED_RR) {
    // row f4, round-robin replicas: 16-byte records only; the recurrence runs up to 2^18 rounds and
    // accumulates the shift of a period, so the state's bound must stay below 2^45 ns
    if (c->N > (u32)MAXN) return fail(c, AUTOPIPE_E_INVAL, "round-robin replicas use 16-byte records: N <= 8");
    if (c->bound >= (1ull << 45))
      return fail(c, AUTOPIPE_E_OVERFLOW, "round-robin replicas need the state's bound below 2^45 ns");
    return AUTOPIPE_OK;
  }
  if ((u128)c->bound * 16u * ((u128)c->model.M + 1) >= ((u128)1 << 63))
    return fail(c, AUTOPIPE_E_OVERFLOW, "16 (M + 1) x the state's bound reaches 2^63 ns");
  return AUTOPIPE_OK;
}

extern "C" int autopipe_set_schedule(autopipe_ctx *c, uint32_t schedule, uint32_t sync, uint32_t micro_batches,
                                     uint32_t flags) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (schedule > AUTOPIPE_SCHED_CHIMERA) return fail(c, AUTOPIPE_E_INVAL, "unknown schedule %u", schedule);
  if (sync > AUTOPIPE_SYNC_PS) return fail(c, AUTOPIPE_E_INVAL, "unknown sync scheme %u", sync);
  if (micro_batches < 1 || micro_batches > AUTOPIPE_MAX_MICRO_BATCHES)
    return fail(c, AUTOPIPE_E_INVAL, "micro_batches = %u outside [1, %u]", micro_batches, AUTOPIPE_MAX_MICRO_BATCHES);
  if ((schedule == AUTOPIPE_SCHED_PIPEDREAM || schedule == AUTOPIPE_SCHED_PIPEDREAM_RR) && micro_batches != 1)
    return fail(c, AUTOPIPE_E_INVAL, "the PipeDream schedules have one mini-batch per iteration (M = 1)");
  if (flags & ~AUTOPIPE_RECOMPUTE) return fail(c, AUTOPIPE_E_INVAL, "unknown flags 0x%x", flags);
  if ((flags & AUTOPIPE_RECOMPUTE) && schedule != AUTOPIPE_SCHED_GPIPE)
    return fail(c, AUTOPIPE_E_INVAL, "AUTOPIPE_RECOMPUTE applies to the GPipe schedule only");
  c->model.sched = schedule;
  c->model.sync = sync;
  c->model.M = micro_batches;
  c->model.recompute = (flags & AUTOPIPE_RECOMPUTE) ? 1u : 0u;
  ++c->gen;
  return AUTOPIPE_OK;
}

extern "C" int autopipe_get_schedule(const autopipe_ctx *c, uint32_t *schedule, uint32_t *sync,
                                     uint32_t *micro_batches, uint32_t *flags) {
  if (!c) return AUTOPIPE_E_INVAL;
  if (schedule) *schedule = c->model.sched;
  if (sync) *sync = c->model.sync;
  if (micro_batches) *micro_batches = c->model.M;
  if (flags) *flags = c->model.recompute ? AUTOPIPE_RECOMPUTE : 0u;
  return AUTOPIPE_OK;
}

static int eval_impl(autopipe_ctx *c, const void *d_parts, uint64_t count, bool wide, uint64_t *d_time_ns,
                     void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "eval before set_state");
  if (count == 0) return AUTOPIPE_OK;
  if (!d_parts || !d_time_ns) return fail(c, AUTOPIPE_E_INVAL, "NULL device pointer");
  DeviceGuard dg(c->device);
  int rc = check_model(c, (cudaStream_t)stream, wide);
  if (rc) return rc;
  // a state given in device memory has not been classified on the host yet: use the 64-bit path
  const int p32 = c->state_on_device ? 0 : (c->path32 | (c->narrow << 1));
  const RRQueue q = rr_queue(c, (cudaStream_t)stream, wide);
  c->launches += launch_eval(c->tab, d_parts, count, wide, (u64 *)d_time_ns, nullptr, nullptr, nullptr, nullptr, p32,
                             c->model, c->sms, next_counter(c), (cudaStream_t)stream, q);
  rr_queue_done(c, (cudaStream_t)stream, q);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "eval kernel launch");
  return AUTOPIPE_OK;
}

extern "C" int autopipe_eval_partitions(autopipe_ctx *c, const autopipe_partition *d_parts, uint64_t count,
                                        uint64_t *d_time_ns, void *stream) {
  return eval_impl(c, d_parts, count, false, d_time_ns, stream);
}

extern "C" int autopipe_eval_partitions_w(autopipe_ctx *c, const autopipe_partition_w *d_parts, uint64_t count,
                                          uint64_t *d_time_ns, void *stream) {
  return eval_impl(c, d_parts, count, true, d_time_ns, stream);
}

// --- search space arithmetic (SPEC.md §5) ----------------------------------------------------
static bool build_space(autopipe_ctx *c, u32 s_min, u32 s_max, u32 flags, SearchSpace &sp) {
  memset(&sp, 0, sizeof(sp));
  sp.L = (int)c->L;
  sp.N = (int)c->N;
  sp.s_min = (int)s_min;
  sp.s_max = (int)s_max;
  sp.flags = (int)(flags & AUTOPIPE_USE_ALL_WORKERS);
  u128 off = 0;
  for (int S = (int)s_min; S <= (int)s_max; ++S) {
    sp.off[S] = (u64)off;
    const u64 K = (flags & AUTOPIPE_USE_ALL_WORKERS) ? c->binom[c->N - 1][S - 1] : c->binom[c->N][S];
    const u64 nc = (S - 1 <= (int)c->L - 1) ? c->binom[c->L - 1][S - 1] : 0;
    if (nc == U64MAX) return false;  // saturated binomial: the space exceeds 2^64
    sp.ncut[S] = nc;
    sp.ncomp[S] = K;
    off += (u128)K * nc;
    if (off >> 64) return false;
  }
  sp.off[s_max + 1] = (u64)off;
  return true;
}

// wide: the space is read through 32-byte records (S <= 16, any N <= 16); otherwise 16-byte records
// (S <= 8 and N <= 8: a contiguous placement may use any of the N workers).
static int check_space_args(autopipe_ctx *c, u32 s_min, u32 s_max, u32 flags, bool wide) {
  if (flags & ~AUTOPIPE_USE_ALL_WORKERS) return fail(c, AUTOPIPE_E_INVAL, "unknown flags 0x%x", flags);
  if (!wide && c->N > (u32)MAXN)
    return fail(c, AUTOPIPE_E_INVAL, "N = %u > 8 workers: 16-byte records cannot name them (use the _w calls)", c->N);
  const u32 lim = wide ? (u32)MAXSW : (u32)MAXS;
  const u32 smax_lim = c->N < lim ? c->N : lim;
  if (s_min < 1 || s_min > s_max || s_max > smax_lim)
    return fail(c, AUTOPIPE_E_INVAL, "need 1 <= s_min <= s_max <= min(%u, N) (got %u, %u, N = %u)", lim, s_min,
                s_max, c->N);
  return AUTOPIPE_OK;
}

extern "C" int autopipe_count_candidates(const autopipe_ctx *cc, uint32_t s_min, uint32_t s_max,
                                         uint32_t flags, uint64_t *total) {
  autopipe_ctx *c = const_cast<autopipe_ctx *>(cc);
  if (!c || !total) return AUTOPIPE_E_INVAL;
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "count before set_state");
  int rc = check_space_args(c, s_min, s_max, flags, true);
  if (rc) return rc;
  SearchSpace sp;
  if (!build_space(c, s_min, s_max, flags, sp)) return fail(c, AUTOPIPE_E_OVERFLOW, "space exceeds 2^64");
  *total = sp.off[s_max + 1];
  return AUTOPIPE_OK;
}

// sorted k-subset (k <= 16) of {0..n-1} of a given lex rank, one element per entry
static void host_unrank(const autopipe_ctx *c, u64 rank, int k, int n, int *out) {
  int x = 0;
  for (int i = 0; i < k; ++i) {
    while (c->binom[n - 1 - x][k - 1 - i] <= rank) {
      rank -= c->binom[n - 1 - x][k - 1 - i];
      ++x;
    }
    out[i] = x++;
  }
}

// Global index -> record bytes (16 or 32 as wide): S, the cuts, the stage of every worker.
static int decode_impl(autopipe_ctx *c, u32 s_min, u32 s_max, u32 flags, u64 index, bool wide, uint8_t *rec) {
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "decode before set_state");
  int rc = check_space_args(c, s_min, s_max, flags, wide);
  if (rc) return rc;
  SearchSpace sp;
  if (!build_space(c, s_min, s_max, flags, sp)) return fail(c, AUTOPIPE_E_OVERFLOW, "space exceeds 2^64");
  if (index >= sp.off[s_max + 1]) return fail(c, AUTOPIPE_E_INVAL, "index beyond the space");
  int S = (int)s_min;
  while (S < (int)s_max && index >= sp.off[S + 1]) ++S;
  const u64 rem = index - sp.off[S];
  const u64 rho = rem / sp.ncut[S], kappa = rem % sp.ncut[S];
  const bool all = flags & AUTOPIPE_USE_ALL_WORKERS;
  int Rp[MAXSW], cuts[MAXSW];
  if (all) host_unrank(c, rho, S - 1, (int)c->N - 1, Rp);
  else host_unrank(c, rho, S, (int)c->N, Rp);
  host_unrank(c, kappa, S - 1, (int)c->L - 1, cuts);
  const int n = wide ? 32 : 16, off = wide ? 16 : 8;
  memset(rec, 0xFF, n);
  rec[0] = (uint8_t)S;
  for (int s = 0; s < S - 1; ++s) rec[1 + s] = (uint8_t)cuts[s];
  int prev = 0;
  for (int s = 0; s < S; ++s) {
    const int R = (all && s == S - 1) ? (int)c->N : Rp[s] + 1;
    for (int w = prev; w < R; ++w) rec[off + w] = (uint8_t)s;
    prev = R;
  }
  return AUTOPIPE_OK;
}

extern "C" int autopipe_decode_index(const autopipe_ctx *cc, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                     uint64_t index, autopipe_partition *out) {
  autopipe_ctx *c = const_cast<autopipe_ctx *>(cc);
  if (!c || !out) return AUTOPIPE_E_INVAL;
  return decode_impl(c, s_min, s_max, flags, index, false, (uint8_t *)out);
}

extern "C" int autopipe_decode_index_w(const autopipe_ctx *cc, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                       uint64_t index, autopipe_partition_w *out) {
  autopipe_ctx *c = const_cast<autopipe_ctx *>(cc);
  if (!c || !out) return AUTOPIPE_E_INVAL;
  return decode_impl(c, s_min, s_max, flags, index, true, (uint8_t *)out);
}

// The search of a 16-byte space (wide = false) or a wide one (row f4). Writes time, index, evaluated
// and the best record (16 or 32 bytes) to the host.
// d_out != nullptr: the asynchronous form (autopipe_search_optimum_async): the result goes to device
// memory on `stream`, nothing waits for the device, and a state set from device memory is not read
// back: the kernels of both integer paths are enqueued and the state kernel's choice gates them.
static int search_impl(autopipe_ctx *c, u32 s_min, u32 s_max, u32 flags, u64 begin, u64 end, bool wide,
                       u64 *h_tie, uint8_t *h_rec, void *stream, void *d_out = nullptr) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  const bool async = d_out != nullptr;
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "search before set_state");
  if (!async && (!h_tie || !h_rec)) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  int rc = check_space_args(c, s_min, s_max, flags, wide);
  if (rc) return rc;
  SearchSpace sp;
  if (!build_space(c, s_min, s_max, flags, sp)) return fail(c, AUTOPIPE_E_OVERFLOW, "space exceeds 2^64");
  const u64 total = sp.off[s_max + 1];
  if (end > total) end = total;
  const int rec_bytes = wide ? 32 : 16;
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  if (!async) {
    h_tie[0] = U64MAX;
    h_tie[1] = U64MAX;
    h_tie[2] = 0;
    memset(h_rec, 0xFF, rec_bytes);
  }
  if (begin >= end) {
    if (async) {  // an empty shard: (UINT64_MAX, UINT64_MAX, 0, record of 0xFF)
      cudaMemsetAsync(d_out, 0xFF, 24 + rec_bytes, st);
      cudaMemsetAsync((unsigned char *)d_out + 16, 0, 8, st);
    }
    return AUTOPIPE_OK;
  }
  // the integer path: known on the host, or (async search of a device state) chosen on the device
  int path = c->path32;
  if (async && c->state_on_device && c->model.sched == SCHED_PIPEDREAM) {
    path = -1;
  } else {
    rc = sync_status(c, st);
    if (rc) return rc;
    rc = check_model(c, st, wide);
    if (rc) return rc;
    path = c->path32;
  }
  if (c->hwork_pending) {  // the pinned schedule slots may still feed the previous search's copies
    cudaEventSynchronize(c->ev_hwork);
    c->hwork_pending = false;
  }
  if (!c->ev_fork) {  // internal streams and events, created once
    cudaError_t e = cudaEventCreateWithFlags(&c->ev_hwork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming);
    for (int i = 0; i < autopipe_ctx::NAUX && e == cudaSuccess; ++i) {
      e = cudaStreamCreateWithFlags(&c->aux[i], cudaStreamNonBlocking);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_join[i], cudaEventDisableTiming);
    }
    if (e != cudaSuccess) return cuda_fail(c, e, "search streams");
  }
  const int tslot = (int)(c->tcount % autopipe_ctx::TRING);
  if (c->timing) cudaEventRecord(c->ev0[tslot], st);
  int used = 0, nlaunch = 0;
  bool forked = false;
  auto next_stream = [&]() -> cudaStream_t {  // fork on first use, then round-robin
    if (!forked) {
      cudaEventRecord(c->ev_fork, st);
      for (int i = 0; i < autopipe_ctx::NAUX; ++i) cudaStreamWaitEvent(c->aux[i], c->ev_fork, 0);
      forked = true;
    }
    return c->aux[(nlaunch++) % autopipe_ctx::NAUX];
  };
  auto join = [&]() {
    if (!forked) return;
    for (int i = 0; i < autopipe_ctx::NAUX; ++i) {
      cudaEventRecord(c->ev_join[i], c->aux[i]);
      cudaStreamWaitEvent(st, c->ev_join[i], 0);
    }
    forked = false;
  };
  // A small range: one dense launch on the caller's stream; a medium PipeDream one: one threshold
  // walk. Otherwise split [begin, end) into the r = 1 block of each S (rho = 0: fast kernel) and the
  // rest (threshold walk or generic); the pieces write disjoint block-result ranges and run
  // concurrently.
  u64 cur = begin;
  if (c->model.sched == SCHED_RR && !wide) {
    // row f4, round-robin replicas: one bound-pruned launch over the whole range plus the drain of
    // its deferred candidates (the deferral queue is the context's; the stream waits for its last user)
    RRQueue q = rr_queue(c, st, false);
    if (!q.buf) {  // AUTOPIPE_RR_NO_DEFER: a queue of capacity 0 (every candidate in its thread)
      cudaStreamWaitEvent(st, c->ev_rrq, 0);
      q.n = c->d_rrq_n;
      q.buf = c->d_rrq;
      q.cap = 0;
    }
    int nb = 0;
    c->launches += launch_search_rr(c->tab, sp, begin, end, c->model, c->sms, c->d_blocks, MAX_BLOCKS, &nb,
                                    next_sched(c), q, st);
    cudaEventRecord(c->ev_rrq, st);
    used = nb;
    cur = end;
  }
  if (cur < end && end - begin <= DENSE_SPAN && !(c->search_options & AUTOPIPE_SEARCH_SPLIT)) {
    int nb = 0;
    // a host-classified state may take the narrow (32-bit stage arithmetic) closed form (bit 1)
    const int dpath = path >= 0 ? (path | (c->narrow << 1)) : path;
    c->launches += launch_search_generic(c->tab, sp, begin, end, dpath, c->model, wide, c->sms, c->d_blocks,
                                         MAX_BLOCKS, &nb, next_sched(c), st, true);
    used = nb;
    cur = end;
  }
#ifndef WALK_SPAN
#define WALK_SPAN (1ull << 28)
#endif
  // a medium PipeDream range (<= 2^28): one threshold-walk launch over all its S, no per-S pieces
  // (B200: BERT-24 state 0.66 -> 0.43 ms, the VGG-16 testbed 1.2 -> 0.36 ms; the 1.3e10-candidate
  // ResNet-50 testbed keeps the per-S split with r = 1 sweeps: 10 ms against 29 ms as one walk)
  if (cur < end && end - begin <= WALK_SPAN && c->model.sched == SCHED_PIPEDREAM &&
      !(c->search_options & AUTOPIPE_SEARCH_SPLIT)) {
    int nb = 0;
    c->launches += launch_search_generic(c->tab, sp, begin, end, path, c->model, wide, c->sms, c->d_blocks,
                                         MAX_BLOCKS, &nb, next_sched(c), st, false);
    used = nb;
    cur = end;
  }
  for (int S = (int)s_min; S <= (int)s_max && cur < end; ++S) {
    const u64 blo = sp.off[S], bhi = sp.off[S + 1];
    if (bhi <= cur) continue;
    const u64 lo = cur, hi = end < bhi ? end : bhi;
    // candidates with rho = 0 are [blo, blo + ncut); rho = 0 is all-r=1 iff the first composition
    // (R = 1..S) has every r_s = 1, which holds for the default flag and for USE_ALL when N = S.
    // The fast kernel decides the PipeDream closed form; other schedules (row f3) go to the generic one.
    const bool r1 = S >= 5 && S <= MAXS && (!(flags & AUTOPIPE_USE_ALL_WORKERS) || (int)c->N == S) &&
                    c->model.sched == SCHED_PIPEDREAM && !(c->search_options & AUTOPIPE_SEARCH_NO_R1);
    const u64 r1hi = blo + sp.ncut[S];
    if (r1 && lo < r1hi) {
      const u64 a = lo, b = hi < r1hi ? hi : r1hi;
      int nb = 0;
      R1Ext ext;
      // the bound only for the state, schedule and space it was seeded on
      if (c->d_bound && c->bound_gen == c->gen && c->bound_key[0] == s_min && c->bound_key[1] == s_max &&
          c->bound_key[2] == flags)
        ext.bound = c->d_bound;
      c->launches += launch_search_r1(c->tab, sp, S, a - blo, b - blo, path, c->sms, c->d_blocks + used,
                                      MAX_BLOCKS - used, &nb, c->d_work, c->h_work, c->work_bytes, next_stream(), ext);
      used += nb;
      if (b < hi) {
        c->launches += launch_search_generic(c->tab, sp, b, hi, path, c->model, wide, c->sms, c->d_blocks + used,
                                             MAX_BLOCKS - used, &nb, next_sched(c), next_stream());
        used += nb;
      }
    } else {
      int nb = 0;
      c->launches += launch_search_generic(c->tab, sp, lo, hi, path, c->model, wide, c->sms, c->d_blocks + used,
                                           MAX_BLOCKS - used, &nb, next_sched(c), next_stream());
      used += nb;
    }
    cur = hi;
    if (used > MAX_BLOCKS - 4 * c->sms) {  // keep room: fold what we have into one entry
      join();
      c->launches += launch_finalize(c->d_blocks, used, sp, c->d_result, wide, st);
      cudaMemcpyAsync(c->d_blocks, c->d_result, sizeof(BlockOut), cudaMemcpyDeviceToDevice, st);
      used = 1;
    }
  }
  join();
  cudaEventRecord(c->ev_hwork, st);
  c->hwork_pending = true;
  if (c->timing) {
    cudaEventRecord(c->ev1[tslot], st);
    ++c->tcount;
  }
  if (experiment_knob("AUTOPIPE_R1_STATS") && used > 0) {  // diagnostics: rare-path decisions per search
    BlockOut *hb = new BlockOut[used];
    cudaMemcpyAsync(hb, c->d_blocks, sizeof(BlockOut) * used, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    u64 rare = 0, cnt = 0;
    for (int i = 0; i < used; ++i) { rare += hb[i].pad; cnt += hb[i].count; }
    fprintf(stderr, "[autopipe] blocks %d candidates %llu rare %llu\n", used, cnt, rare);
    delete[] hb;
  }
  if (async) {
    c->launches += launch_finalize(c->d_blocks, used, sp, (ResultDev *)d_out, wide, st, rec_bytes);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(c, e, "search kernel launch");
    return AUTOPIPE_OK;
  }
  c->launches += launch_finalize(c->d_blocks, used, sp, c->d_result, wide, st);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "search kernel launch");
  e = cudaMemcpyAsync(c->h_result, c->d_result, sizeof(ResultDev), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(c, e, "search");
  c->hwork_pending = false;
  h_tie[0] = c->h_result->time_ns;
  h_tie[1] = c->h_result->index;
  h_tie[2] = c->h_result->evaluated;
  memcpy(h_rec, c->h_result->part, wide ? 32 : 16);
  return AUTOPIPE_OK;
}

// Row e, cross-shard bound: the seed half of a search. For every r = 1 block of [begin, end) with at
// least 2^26 candidates, the seed kernel finds a good candidate of the shard; its exact T is
// min-folded into *d_theta (set to UINT64_MAX first). Nothing else runs: no sweep, no result.
extern "C" int autopipe_search_seed_async(autopipe_ctx *c, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                          uint64_t begin, uint64_t end, uint64_t *d_theta, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!d_theta) return fail(c, AUTOPIPE_E_INVAL, "NULL theta pointer");
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "seed before set_state");
  int rc = check_space_args(c, s_min, s_max, flags, false);
  if (rc) return rc;
  SearchSpace sp;
  if (!build_space(c, s_min, s_max, flags, sp)) return fail(c, AUTOPIPE_E_OVERFLOW, "space exceeds 2^64");
  const u64 total = sp.off[s_max + 1];
  if (end > total) end = total;
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  c->seed_gen = c->gen;
  c->seed_key[0] = s_min; c->seed_key[1] = s_max; c->seed_key[2] = flags;
  cudaError_t e = cudaMemsetAsync(d_theta, 0xFF, sizeof(u64), st);
  if (e != cudaSuccess) return cuda_fail(c, e, "seed");
  if (!c->ev_hseed) {
    e = cudaEventCreateWithFlags(&c->ev_hseed, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(c, e, "seed event");
  }
  if (c->hseed_pending) {  // the pinned slots may still feed the previous seed call's copies
    cudaEventSynchronize(c->ev_hseed);
    c->hseed_pending = false;
  }
  const size_t half = c->work_bytes / 2;
  void *dw = (unsigned char *)c->d_work + half, *hw = (unsigned char *)c->h_work + half;
  for (int S = (int)s_min; S <= (int)s_max && begin < end; ++S) {
    const u64 blo = sp.off[S], r1hi = blo + sp.ncut[S];
    const bool r1 = S >= 5 && S <= MAXS && (!(flags & AUTOPIPE_USE_ALL_WORKERS) || (int)c->N == S) &&
                    c->model.sched == SCHED_PIPEDREAM;
    const u64 a = begin > blo ? begin : blo, b = end < r1hi ? end : r1hi;
    if (!r1 || a >= b) continue;
    R1Ext ext;
    ext.theta_out = (u64 *)d_theta;
    int nb = 0;
    c->launches += launch_search_r1(c->tab, sp, S, a - blo, b - blo, 0, c->sms, c->d_blocks, MAX_BLOCKS, &nb, dw, hw,
                                    half, st, ext);
  }
  cudaEventRecord(c->ev_hseed, st);
  c->hseed_pending = true;
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "seed kernel launch");
  return AUTOPIPE_OK;
}

extern "C" int autopipe_set_search_bound(autopipe_ctx *c, const uint64_t *d_bound) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!d_bound) {
    c->d_bound = nullptr;
    c->bound_gen = ~0ull;
    return AUTOPIPE_OK;
  }
  if (c->seed_gen != c->gen)
    return fail(c, AUTOPIPE_E_STATE, "no seed call on the current profile, state and schedule");
  c->d_bound = (const u64 *)d_bound;
  c->bound_gen = c->seed_gen;
  memcpy(c->bound_key, c->seed_key, sizeof(c->bound_key));
  return AUTOPIPE_OK;
}

extern "C" int autopipe_search_optimum(autopipe_ctx *c, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                       uint64_t begin, uint64_t end, autopipe_result *h_out, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  if (!h_out) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  u64 tie[3];
  const int rc = search_impl(c, s_min, s_max, flags, begin, end, false, tie, (uint8_t *)&h_out->part, stream);
  h_out->time_ns = tie[0];
  h_out->index = tie[1];
  h_out->evaluated = tie[2];
  return rc;
}

extern "C" int autopipe_search_optimum_async(autopipe_ctx *c, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                             uint64_t begin, uint64_t end, autopipe_result *d_out, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  if (!d_out) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  return search_impl(c, s_min, s_max, flags, begin, end, false, nullptr, nullptr, stream, d_out);
}

extern "C" int autopipe_search_optimum_async_w(autopipe_ctx *c, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                               uint64_t begin, uint64_t end, autopipe_result_w *d_out, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  if (!d_out) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  return search_impl(c, s_min, s_max, flags, begin, end, true, nullptr, nullptr, stream, d_out);
}

extern "C" int autopipe_reduce_results(const autopipe_result *d_in, uint32_t n, autopipe_result *d_out,
                                       void *stream) {
  if (!d_out || (n > 0 && !d_in)) return AUTOPIPE_E_INVAL;
  launch_reduce_results(d_in, n, 16, d_out, (cudaStream_t)stream);
  return cudaGetLastError() == cudaSuccess ? AUTOPIPE_OK : AUTOPIPE_E_CUDA;
}

extern "C" int autopipe_reduce_results_w(const autopipe_result_w *d_in, uint32_t n, autopipe_result_w *d_out,
                                         void *stream) {
  if (!d_out || (n > 0 && !d_in)) return AUTOPIPE_E_INVAL;
  launch_reduce_results(d_in, n, 32, d_out, (cudaStream_t)stream);
  return cudaGetLastError() == cudaSuccess ? AUTOPIPE_OK : AUTOPIPE_E_CUDA;
}

extern "C" int autopipe_search_optimum_w(autopipe_ctx *c, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                         uint64_t begin, uint64_t end, autopipe_result_w *h_out, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  if (!h_out) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  u64 tie[3];
  const int rc = search_impl(c, s_min, s_max, flags, begin, end, true, tie, (uint8_t *)&h_out->part, stream);
  h_out->time_ns = tie[0];
  h_out->index = tie[1];
  h_out->evaluated = tie[2];
  return rc;
}

// host-side validation of a current partition (same rules as SPEC.md §2), 16-byte (MS = 8) or wide
// (MS = 16) record bytes; its packed parts as the kernels read them (P8: cuts[0], masks[0]; P16:
// cut bytes in cuts[0..1], 16-bit stage masks in masks[0..3]).
static bool host_decode_rec(const uint8_t *rec, bool wide, u32 L, u32 N, int &S, u64 *cuts, u64 *masks) {
  const int MS = wide ? MAXSW : MAXS, off = wide ? 16 : 8, mb = wide ? 16 : 8;
  S = rec[0];
  if (S < 1 || S > MS || S > (int)N) return false;
  cuts[0] = cuts[1] = 0;
  for (int i = 0; i < 4; ++i) masks[i] = 0;
  int prev = -1;
  for (int i = 0; i < S - 1; ++i) {
    const int e = rec[1 + i];
    if (e <= prev || e >= (int)L - 1) return false;
    prev = e;
    cuts[i >> 3] |= (u64)e << (8 * (i & 7));
  }
  u32 sm[MAXSW] = {0};
  for (int w = 0; w < MS; ++w) {
    const int s = rec[off + w];
    if (s == 0xFF) continue;
    if (w >= (int)N || s >= S) return false;
    sm[s] |= 1u << w;
  }
  for (int s = 0; s < S; ++s) {
    if (sm[s] == 0) return false;
    if (wide) masks[s >> 2] |= (u64)sm[s] << (16 * (s & 3));
    else masks[0] |= (u64)sm[s] << (mb * s);
  }
  return true;
}
static bool host_decode(const autopipe_partition *p, u32 L, u32 N, int &S, u64 &cuts, u64 &masks) {
  u64 c2[2], m4[4];
  if (!host_decode_rec((const uint8_t *)p, false, L, N, S, c2, m4)) return false;
  cuts = c2[0];
  masks = m4[0];
  return true;
}

static int rollout_impl(autopipe_ctx *c, const void *d_parts, uint64_t count, const uint8_t *h_current, bool wide,
                        uint64_t *d_time_ns, uint64_t *d_switch_bytes, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "rollout before set_state");
  if ((h_current == nullptr) != (d_switch_bytes == nullptr))
    return fail(c, AUTOPIPE_E_INVAL, "h_current and d_switch_bytes must both be set or both be NULL");
  int S = 0;
  u64 cuts[2], masks[4];
  if (h_current && !host_decode_rec(h_current, wide, c->L, c->N, S, cuts, masks))
    return fail(c, AUTOPIPE_E_INVAL, "invalid current partition");
  if (count == 0) return AUTOPIPE_OK;
  if (!d_parts || !d_time_ns) return fail(c, AUTOPIPE_E_INVAL, "NULL device pointer");
  DeviceGuard dg(c->device);
  int rc = check_model(c, (cudaStream_t)stream, wide);
  if (rc) return rc;
  const int p32 = c->state_on_device ? 0 : (c->path32 | (c->narrow << 1));
  const RRQueue q = rr_queue(c, (cudaStream_t)stream, wide);
  c->launches += launch_eval(c->tab, d_parts, count, wide, (u64 *)d_time_ns, (u64 *)d_switch_bytes,
                             h_current ? &S : nullptr, cuts, masks, p32, c->model, c->sms, next_counter(c),
                             (cudaStream_t)stream, q);
  rr_queue_done(c, (cudaStream_t)stream, q);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "rollout kernel launch");
  return AUTOPIPE_OK;
}

extern "C" int autopipe_rollout_rewards(autopipe_ctx *c, const autopipe_partition *d_parts, uint64_t count,
                                        const autopipe_partition *h_current, uint64_t *d_time_ns,
                                        uint64_t *d_switch_bytes, void *stream) {
  return rollout_impl(c, d_parts, count, (const uint8_t *)h_current, false, d_time_ns, d_switch_bytes, stream);
}

extern "C" int autopipe_rollout_rewards_w(autopipe_ctx *c, const autopipe_partition_w *d_parts, uint64_t count,
                                          const autopipe_partition_w *h_current, uint64_t *d_time_ns,
                                          uint64_t *d_switch_bytes, void *stream) {
  return rollout_impl(c, d_parts, count, (const uint8_t *)h_current, true, d_time_ns, d_switch_bytes, stream);
}

extern "C" int autopipe_int_path(const autopipe_ctx *cc) {
  autopipe_ctx *c = const_cast<autopipe_ctx *>(cc);
  if (!c || !c->has_state) return 0;
  DeviceGuard dg(c->device);
  cudaDeviceSynchronize();
  if (sync_status(c, nullptr)) return 0;
  return c->path32 ? 32 : 64;
}

extern "C" uint64_t autopipe_kernel_launches(const autopipe_ctx *c) { return c ? c->launches : 0; }

extern "C" int autopipe_set_search_options(autopipe_ctx *c, uint32_t options) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (options & ~(AUTOPIPE_SEARCH_SPLIT | AUTOPIPE_SEARCH_NO_R1 | AUTOPIPE_RR_DEFER_ALL | AUTOPIPE_RR_NO_DEFER))
    return fail(c, AUTOPIPE_E_INVAL, "unknown search options 0x%x", options);
  c->search_options = options;
  return AUTOPIPE_OK;
}

extern "C" int autopipe_set_timing(autopipe_ctx *c, int enable) {
  if (!c) return AUTOPIPE_E_INVAL;
  DeviceGuard dg(c->device);
  if (enable && !c->ev0[0]) {
    for (int i = 0; i < autopipe_ctx::TRING; ++i) {
      cudaError_t e = cudaEventCreate(&c->ev0[i]);
      if (e == cudaSuccess) e = cudaEventCreate(&c->ev1[i]);
      if (e != cudaSuccess) return cuda_fail(c, e, "event create");
    }
  }
  c->timing = enable != 0;
  return AUTOPIPE_OK;
}

static double pair_ms(autopipe_ctx *c, u64 k) {
  const int i = (int)(k % autopipe_ctx::TRING);
  float ms = 0.f;
  cudaEventSynchronize(c->ev1[i]);
  if (cudaEventElapsedTime(&ms, c->ev0[i], c->ev1[i]) != cudaSuccess) return -1.0;
  return ms;
}

extern "C" double autopipe_last_search_ms(const autopipe_ctx *cc) {
  autopipe_ctx *c = const_cast<autopipe_ctx *>(cc);
  if (!c || c->tcount == 0) return -1.0;
  DeviceGuard dg(c->device);
  return pair_ms(c, c->tcount - 1);
}

extern "C" int autopipe_search_times(autopipe_ctx *c, double *ms, uint32_t cap, uint32_t *count) {
  if (!c || !count || (cap > 0 && !ms)) return AUTOPIPE_E_INVAL;
  DeviceGuard dg(c->device);
  u64 k = c->tread;
  if (c->tcount - k > (u64)autopipe_ctx::TRING) k = c->tcount - autopipe_ctx::TRING;  // older pairs reused
  uint32_t n = 0;
  for (; k < c->tcount && n < cap; ++k) ms[n++] = pair_ms(c, k);
  c->tread = k;
  *count = n;
  return AUTOPIPE_OK;
}

// --- NEXT row f1: the two-worker neighbourhood (reading F-1) ----------------
static int neigh_prepare(autopipe_ctx *c, const autopipe_partition *h_current, u64 &nslots, cudaStream_t st) {
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "neighbourhood before set_state");
  if (!h_current) return fail(c, AUTOPIPE_E_INVAL, "NULL current partition");
  if (c->N > (u32)MAXN) return fail(c, AUTOPIPE_E_INVAL, "the neighbourhood uses 16-byte records: N <= 8");
  int S = 0;
  u64 cuts = 0, masks = 0;
  if (!host_decode(h_current, c->L, c->N, S, cuts, masks))
    return fail(c, AUTOPIPE_E_INVAL, "invalid current partition");
  u64 sow = 0;
  for (int w = 0; w < MAXN; ++w) sow |= (u64)h_current->stage_of_worker[w] << (8 * w);
  nslots = (u64)((int)c->N + (int)c->N * ((int)c->N - 1) / 2) * NEIGH_MAXOPT;
  c->launches += launch_neigh_gen(S, cuts, sow, (int)c->L, (int)c->N, c->d_nslots, st);
  return AUTOPIPE_OK;
}

extern "C" int autopipe_neighbourhood(autopipe_ctx *c, const autopipe_partition *h_current, autopipe_partition *d_out,
                                      uint64_t capacity, uint64_t *h_count, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!h_count || (capacity && !d_out)) return fail(c, AUTOPIPE_E_INVAL, "NULL output");
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  u64 nslots = 0;
  int rc = neigh_prepare(c, h_current, nslots, st);
  if (rc) return rc;
  c->launches += launch_neigh_compact(c->d_nslots, nslots, d_out, capacity, c->d_ncount, st);
  cudaError_t e = cudaMemcpyAsync(c->h_ncount, c->d_ncount, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(c, e, "neighbourhood");
  *h_count = *c->h_ncount;
  return AUTOPIPE_OK;
}

extern "C" int autopipe_neighbourhood_best(autopipe_ctx *c, const autopipe_partition *h_current,
                                           autopipe_result *h_out, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!h_out) return fail(c, AUTOPIPE_E_INVAL, "NULL result pointer");
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  int rc = sync_status(c, st);
  if (rc) return rc;
  rc = check_model(c, st);
  if (rc) return rc;
  u64 nslots = 0;
  rc = neigh_prepare(c, h_current, nslots, st);
  if (rc) return rc;
  c->launches += launch_eval(c->tab, c->d_nslots, nslots, false, c->d_ntimes, nullptr, nullptr, nullptr, nullptr,
                             c->path32, c->model, c->sms, next_counter(c), st);
  c->launches += launch_neigh_best(c->d_nslots, c->d_ntimes, nslots, c->d_result, st);
  cudaError_t e = cudaMemcpyAsync(c->h_result, c->d_result, sizeof(ResultDev), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(c, e, "neighbourhood_best");
  h_out->time_ns = c->h_result->time_ns;
  h_out->index = c->h_result->index;
  h_out->evaluated = c->h_result->evaluated;
  memcpy(&h_out->part, c->h_result->part, 16);
  return AUTOPIPE_OK;
}

// The paper's gradual migration: from *h_start, move to the best two-worker
// neighbour while it is strictly faster. Every score comes from the eval kernel; the loop runs here.
extern "C" int autopipe_local_search(autopipe_ctx *c, const autopipe_partition *h_start, uint32_t max_steps,
                                     autopipe_result *h_path, uint32_t capacity, uint32_t *h_count, void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!h_start || !h_path || !h_count || capacity == 0) return fail(c, AUTOPIPE_E_INVAL, "NULL pointer or zero capacity");
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "local search before set_state");
  if (c->N > (u32)MAXN) return fail(c, AUTOPIPE_E_INVAL, "the neighbourhood uses 16-byte records: N <= 8");
  int S = 0;
  u64 cuts = 0, masks = 0;
  if (!host_decode(h_start, c->L, c->N, S, cuts, masks)) return fail(c, AUTOPIPE_E_INVAL, "invalid start partition");
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  int rc = sync_status(c, st);
  if (rc) return rc;
  rc = check_model(c, st);
  if (rc) return rc;
  // T of the start: one record through the eval kernel (slot 0 of the neighbourhood area)
  cudaError_t e = cudaMemcpyAsync(c->d_nslots, h_start, 16, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return cuda_fail(c, e, "local search");
  c->launches += launch_eval(c->tab, c->d_nslots, 1, false, c->d_ntimes, nullptr, nullptr, nullptr, nullptr, c->path32,
                             c->model, c->sms, next_counter(c), st);
  e = cudaMemcpyAsync(&c->h_result->time_ns, c->d_ntimes, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(c, e, "local search");
  h_path[0].time_ns = c->h_result->time_ns;
  h_path[0].index = U64MAX;
  h_path[0].evaluated = 1;
  memcpy(&h_path[0].part, h_start, 16);
  uint32_t n = 1;
  for (uint32_t step = 0; step < max_steps && n < capacity; ++step) {
    autopipe_result r;
    rc = autopipe_neighbourhood_best(c, &h_path[n - 1].part, &r, stream);
    if (rc) return rc;
    if (r.time_ns >= h_path[n - 1].time_ns) break;  // no strictly faster neighbour: a local optimum
    h_path[n++] = r;
  }
  *h_count = n;
  return AUTOPIPE_OK;
}

// --- NEXT row f2: switching cost as time (reading F-2) ----
static const u64 LIMIT_SWITCH = 1ull << 52;  // startup event times < 2^10 * bound (DESIGN.md §3 F-2)

extern "C" int autopipe_switch_rewards(autopipe_ctx *c, const autopipe_partition *d_parts, uint64_t count,
                                       const autopipe_partition *h_current, uint64_t horizon, uint64_t *d_time_ns,
                                       uint64_t *d_refill_ns, uint64_t *d_migrate_ns, uint64_t *d_reward_ns,
                                       void *stream) {
  if (!c) return AUTOPIPE_E_INVAL;
  c->err[0] = 0;
  if (!c->has_state) return fail(c, AUTOPIPE_E_STATE, "switch rewards before set_state");
  if (!h_current) return fail(c, AUTOPIPE_E_INVAL, "NULL current partition");
  if (horizon == 0) return fail(c, AUTOPIPE_E_INVAL, "horizon must be >= 1");
  if (c->N > (u32)MAXN) return fail(c, AUTOPIPE_E_INVAL, "switch rewards use 16-byte records: N <= 8");
  if (c->model.sched != SCHED_PIPEDREAM)
    return fail(c, AUTOPIPE_E_STATE, "switch rewards are defined for the PipeDream schedule (reading F-2)");
  int S = 0;
  u64 cuts = 0, masks = 0;
  if (!host_decode(h_current, c->L, c->N, S, cuts, masks))
    return fail(c, AUTOPIPE_E_INVAL, "invalid current partition");
  if (count == 0) return AUTOPIPE_OK;
  if (!d_parts || !d_reward_ns) return fail(c, AUTOPIPE_E_INVAL, "NULL device pointer");
  DeviceGuard dg(c->device);
  cudaStream_t st = (cudaStream_t)stream;
  int rc = sync_status(c, st);
  if (rc) return rc;
  if (c->bound >= LIMIT_SWITCH)
    return fail(c, AUTOPIPE_E_OVERFLOW, "switch rewards need modelled times below 2^52 ns");
  u64 sow = 0;
  for (int w = 0; w < MAXN; ++w) sow |= (u64)h_current->stage_of_worker[w] << (8 * w);
  c->launches += launch_switch(c->tab, d_parts, count, S, cuts, masks, sow, horizon, (u64 *)d_time_ns,
                               (u64 *)d_refill_ns, (u64 *)d_migrate_ns, (u64 *)d_reward_ns, c->path32, (int)c->model.sync,
                               c->sms, next_counter(c), st);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "switch kernel launch");
  return AUTOPIPE_OK;
}

// --- cost-balanced contiguous shards of a search space ---------------
// Estimated device cost (thread-instructions per lane) of the r = 1 kernel: a row (prefix, y) costs
// ROW + X * (m - 1) + CAND * m (m - 1) / 2 with m = L - 2 - y (calibrated on B200: the per-row term
// is what makes the high-index shards, whose rows are short, slower per candidate; re-fitted with
// the seeded sweep: max/min of 8 C(95,7) shards 1.07 (C4a), 1.05 (C4b)); the generic
// kernel costs GEN * S per candidate.
namespace {
// per-row fixed cost of the r = 1 sweep: the 64-bit path (the default), and the 32-bit one, whose
// candidates are cheaper against the same per-row work (B200, the 96-layer 8-stage space, slowest of
// 8 shards: C4a 0.499 ms at 600, 0.479 at 1000; C4b 0.652 at 600, 0.669 at 1000)
const u64 COST_ROW = 600, COST_ROW32 = 1000, COST_X = 30, COST_CAND = 4, COST_GEN = 40;
u64 hbin[256][17];  // C(n, k), k <= 16 (wide spaces), saturated at 2^64 - 1
void hbin_init() {
  static bool done = false;
  if (done) return;
  for (int n = 0; n < 256; ++n)
    for (int k = 0; k < 17; ++k) {
      const u64 a = (n == 0) ? 0 : hbin[n - 1][k - (k > 0)], b = (n == 0) ? 0 : hbin[n - 1][k];
      hbin[n][k] = (k == 0) ? 1 : (a + b < a ? ~0ull : a + b);
    }
  done = true;
}
inline u64 hbn(int n, int k) { return (k < 0 || n < 0 || k > n) ? 0 : hbin[n][k]; }
void unrank_cuts(u64 rank, int k, int n, int *out) {
  int x = 0;
  for (int i = 0; i < k; ++i) {
    while (hbn(n - 1 - x, k - 1 - i) <= rank) {
      rank -= hbn(n - 1 - x, k - 1 - i);
      ++x;
    }
    out[i] = x++;
  }
}
// k-subsets of {0..x-1} lexicographically smaller than the increasing tuple t
u64 count_less_t(int x, int k, const int *t) {
  u64 cnt = 0;
  int prev = -1;
  for (int i = 0; i < k; ++i) {
    const int lim = t[i] < x ? t[i] : x;
    for (int v = prev + 1; v < lim; ++v) cnt += hbn(x - 1 - v, k - 1 - i);
    if (t[i] >= x) return cnt;
    prev = t[i];
  }
  return cnt;
}
inline double row_cost(int L, int y, double row) {
  // AUTOPIPE_COST_{ROW,X,CAND}: experiment knobs for re-fitting the model (unset: the constants)
  static const char *kr = experiment_knob("AUTOPIPE_COST_ROW"), *kx = experiment_knob("AUTOPIPE_COST_X"),
                    *kc = experiment_knob("AUTOPIPE_COST_CAND");
  const double cr = kr ? atof(kr) : row;
  static const double cx = kx ? atof(kx) : (double)COST_X;
  static const double cc = kc ? atof(kc) : (double)COST_CAND;
  const double m = (double)(L - 2 - y);
  return cr + cx * (m - 1) + cc * m * (m - 1) / 2;
}
// cost of the first `kappa` cut sets (lexicographic) of an r = 1 block with S stages
double r1_prefix_cost(int L, int S, u64 kappa, u64 ncut, double row) {
  if (kappa == 0) return 0.0;
  const int P = S - 4, n = L - 1, k = S - 1;
  int lo[8];
  const bool end = kappa >= ncut;
  unrank_cuts(end ? ncut - 1 : kappa, k, n, lo);
  double c = 0.0;
  for (int y = P; y <= L - 4; ++y) {
    const bool fits = (P == 0) || lo[P - 1] < y;
    u64 rows = count_less_t(y, P, lo) + ((fits && y < lo[P]) ? 1 : 0);
    if (end && fits && y == lo[P]) rows += 1;  // the last row itself
    c += (double)rows * row_cost(L, y, row);
  }
  return c;
}
}  // namespace

static int balanced_shards(uint32_t L, uint32_t N, uint32_t s_min, uint32_t s_max, uint32_t flags, uint32_t G,
                           double row, uint64_t *bounds) {
  if (!bounds || G < 1 || L < 1 || L > MAXL || N < 1 || N > MAXNW) return AUTOPIPE_E_INVAL;
  if (flags & ~AUTOPIPE_USE_ALL_WORKERS) return AUTOPIPE_E_INVAL;
  // 16-byte spaces (S, N <= 8) and wide ones (row f4: S, N <= 16; their S > 8 blocks are generic)
  const u32 smax_lim = N < (u32)MAXSW ? N : (u32)MAXSW;
  if (s_min < 1 || s_min > s_max || s_max > smax_lim) return AUTOPIPE_E_INVAL;
  hbin_init();
  const bool all = flags & AUTOPIPE_USE_ALL_WORKERS;
  // blocks of the index space in order: per S, the r = 1 block (if the fast kernel takes it) and the rest
  struct Blk { u64 lo, hi; int S; bool r1; double c0, c1; };
  Blk blk[2 * MAXS];
  int nb = 0;
  u128 off = 0;
  double acc = 0.0;
  for (int S = (int)s_min; S <= (int)s_max; ++S) {
    const u64 K = all ? hbn((int)N - 1, S - 1) : hbn((int)N, S);
    const u64 nc = (S - 1 <= (int)L - 1) ? hbn((int)L - 1, S - 1) : 0;
    const u128 sz = (u128)K * nc;
    if ((off + sz) >> 64) return AUTOPIPE_E_OVERFLOW;
    const bool r1 = S >= 5 && S <= MAXS && (!all || (int)N == S) && nc > 0;
    u64 start = (u64)off;
    if (r1) {
      const double c = r1_prefix_cost((int)L, S, nc, nc, row);
      blk[nb++] = {start, start + nc, S, true, acc, acc + c};
      acc += c;
      start += nc;
    }
    const u64 rest = (u64)(off + sz) - start;
    if (rest) {
      const double c = (double)rest * COST_GEN * S;
      blk[nb++] = {start, start + rest, S, false, acc, acc + c};
      acc += c;
    }
    off += sz;
  }
  const u64 total = (u64)off;
  bounds[0] = 0;
  bounds[G] = total;
  for (u32 g = 1; g < G; ++g) {
    const double target = acc * (double)g / (double)G;
    u64 b = total;
    for (int i = 0; i < nb; ++i) {
      if (target > blk[i].c1) continue;
      const Blk &B = blk[i];
      if (!B.r1) {
        const double f = (B.c1 > B.c0) ? (target - B.c0) / (B.c1 - B.c0) : 0.0;
        b = B.lo + (u64)(f * (double)(B.hi - B.lo));
      } else {  // bisection on the cut rank: the prefix cost is monotone
        u64 a = 0, z = B.hi - B.lo;
        while (a < z) {
          const u64 mid = a + (z - a) / 2;
          if (B.c0 + r1_prefix_cost((int)L, B.S, mid, B.hi - B.lo, row) < target) a = mid + 1;
          else z = mid;
        }
        b = B.lo + a;
      }
      break;
    }
    if (b < bounds[g - 1]) b = bounds[g - 1];
    if (b > total) b = total;
    bounds[g] = b;
  }
  return AUTOPIPE_OK;
}

extern "C" int autopipe_balanced_shards(uint32_t L, uint32_t N, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                        uint32_t G, uint64_t *bounds) {
  return balanced_shards(L, N, s_min, s_max, flags, G, (double)COST_ROW, bounds);
}

extern "C" int autopipe_balanced_shards_path(uint32_t L, uint32_t N, uint32_t s_min, uint32_t s_max, uint32_t flags,
                                             uint32_t G, uint32_t int_path, uint64_t *bounds) {
  if (int_path != 32 && int_path != 64) return AUTOPIPE_E_INVAL;
  return balanced_shards(L, N, s_min, s_max, flags, G, (double)(int_path == 32 ? COST_ROW32 : COST_ROW), bounds);
}
