// k_search_r1.cu — fast exhaustive search over the r = 1 block of one S (placeholder: generic path).
#include "internal.h"

namespace ap {

int launch_search_r1(const DevTables &g, const SearchSpace &sp, int S, u64 k_begin, u64 k_end, int path32,
                     int sms, BlockOut *out, int max_blocks, int *nblocks, void *work, size_t work_bytes,
                     cudaStream_t st) {
  (void)path32; (void)work; (void)work_bytes;
  return launch_search_generic(g, sp, sp.off[S] + k_begin, sp.off[S] + k_end, sms, out, max_blocks, nblocks, st);
}

}  // namespace ap
