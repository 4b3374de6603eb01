// kernels.cu — the single device translation unit (one copy of the __constant__ binomial table).
#include "binom.cuh"
#include "k_state.cu"
#include "k_eval.cu"
#include "k_search.cu"
#include "k_search_r1.cu"
#include "k_neigh.cu"
#include "k_switch.cu"
