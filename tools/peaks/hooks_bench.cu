// Microbenchmarks of the hook building blocks on the B200 (informs DESIGN.md §5):
//   sectors_lines() (monotone fast path / 32-bit sort / 64-bit sort) vs __match_any_sync, per address
//   pattern; shared-memory red.add.u32 throughput with scattered addresses.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I../../include
//             -I../../paper_conf_micro_villasnk19_b200/csrc -o hooks_bench hooks_bench.cu
#include <cstdio>
#include <cstdlib>
#include "nvbt_hooks.cuh"

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e_), __LINE__); exit(1);} } while (0)
using namespace nvbt;

__device__ __forceinline__ unsigned long long pattern_addr(int pat, unsigned lane, unsigned long long x) {
  const unsigned long long base = (x & ((1ull << 40) - 1)) & ~127ull;
  switch (pat) {
    case 0: return base + lane * 4;                       // coalesced
    case 1: return base + lane * 4096;                    // strided (SGEMM A)
    case 2: return base;                                  // broadcast
    case 3: return base + (((x >> 7) * (lane + 1) * 2654435761u) & 1023) * 4;  // random in 4 KB
    case 4: return ((x * (lane + 7) * 0x9E3779B97F4A7C15ull) & ((1ull << 40) - 1)) & ~3ull;  // random 2^40
    default: return base + (lane ^ 13) * 4;               // lane-XOR permuted
  }
}

template <int MODE>
__global__ void k_div(int pat, int iters, unsigned* out) {
  const unsigned lane = lane_id(), lanebit = 1u << lane, lmlt = lanemask_lt();
  __shared__ unsigned scr_all[8 * SCRATCH_WORDS];
  for (int i = threadIdx.x; i < 8 * SCRATCH_WORDS; i += blockDim.x) scr_all[i] = scratch_init_word(i % SCRATCH_WORDS);
  __syncthreads();
  const unsigned bm = (unsigned)__cvta_generic_to_shared(scr_all + SCRATCH_WORDS * (threadIdx.x >> 5));
  unsigned acc = 0;
  unsigned long long x = 0x1234567ull * (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  for (int i = 0; i < iters; ++i) {
    x = x * 6364136223846793005ull + 1442695040888963407ull;
    const unsigned long long xu = __shfl_sync(FULL, x, 0);
    const unsigned long long a = pattern_addr(pat, lane, xu);
    const unsigned E = 0xffffffffu;
    unsigned S, L;
    if (MODE == 0) {
      sectors_lines<true>(a, E, lane, lanebit, lmlt, bm, S, L);
    } else {
      S = distinct_match(a >> 5, E, lanebit, lmlt);
      L = distinct_match(a >> 7, E, lanebit, lmlt);
    }
    acc += S * 33 + L;
  }
  if (acc == 0x7fffffff) out[0] = acc;
}

__global__ void k_red(int iters, unsigned* out, int spread) {
  __shared__ unsigned bins[2 * 4096];
  for (int i = threadIdx.x; i < 2 * 4096; i += blockDim.x) bins[i] = 0;
  __syncthreads();
  const unsigned sb = (unsigned)__cvta_generic_to_shared(bins);
  unsigned x = threadIdx.x * 2654435761u + blockIdx.x * 97u;
  for (int i = 0; i < iters; ++i) {
    x = x * 1664525u + 1013904223u;
    const unsigned pc = spread ? (x >> 12) & 4095 : (x >> 12) & 7;
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(sb + 4 * pc), "r"((x >> 3) & 31) : "memory");
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(sb + 4 * (4096 + pc)), "r"(1u) : "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0 && bins[5] == 0x7fffffff) out[0] = 1;
}

int main() {
  unsigned* out;
  CK(cudaMalloc(&out, 64));
  int sms = 148;
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  const char* names[] = {"coalesced", "strided4096", "broadcast", "random4K", "random2^40", "xor"};
  const int iters = 2048;
  printf("{");
  for (int mode = 0; mode < 2; ++mode) {
    for (int pat = 0; pat < 6; ++pat) {
      auto launch = [&]() {
        if (mode == 0) k_div<0><<<sms * 4, 256>>>(pat, iters, out);
        else k_div<1><<<sms * 4, 256>>>(pat, iters, out);
      };
      launch(); CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(a)); launch(); CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
      float ms; CK(cudaEventElapsedTime(&ms, a, b));
      const double ops = (double)sms * 4 * 8 * iters;  // warp-events
      // SM-cycles per warp-event at 1.965 GHz
      printf("%s\"%s_%s_Gev_s\": %.2f, \"%s_%s_smcyc_per_ev\": %.1f", (mode || pat) ? ", " : "",
             mode ? "match" : "sort", names[pat], ops / (ms * 1e6), mode ? "match" : "sort", names[pat],
             ms * 1e-3 * 1.965e9 * sms / ops);
    }
  }
  for (int spread = 0; spread < 2; ++spread) {
    const int it = 4096;
    k_red<<<sms * 2, 1024>>>(it, out, spread); CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(a)); k_red<<<sms * 2, 1024>>>(it, out, spread); CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    const double lanes = (double)sms * 2 * 1024 * it * 2;
    printf(", \"red_shared_%s_Glane_s\": %.1f, \"red_shared_%s_lanes_per_smclk\": %.2f", spread ? "4096bins" : "8bins",
           lanes / (ms * 1e6), spread ? "4096bins" : "8bins", lanes / (ms * 1e-3 * 1.965e9 * sms));
  }
  printf("}\n");
  return 0;
}
