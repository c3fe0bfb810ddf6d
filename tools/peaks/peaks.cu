// Box microbenchmarks for the nvbt rooflines.
// Measures the primitive rates the hot path is built from, on the B200 it runs on:
//   MATCH.ANY.U64 / VOTE+POPC issue rate, shared-memory atomics (u32/u64, spread),
//   global RED.ADD.U64 (same address / distinct), HBM read-only bandwidth,
//   D2H link bandwidth (copy engine; SM stores into mapped pinned memory; bulk copy).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o peaks peaks.cu
// Output: one JSON object on stdout.
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1);} } while (0)

static int g_sms = 0;
static float time_kernel(void (*launch)(void*), void* arg, int reps = 5) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  launch(arg); CK(cudaDeviceSynchronize());
  float best = 1e30f;
  for (int r = 0; r < reps; ++r) {
    CK(cudaEventRecord(a)); launch(arg); CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b)); if (ms < best) best = ms;
  }
  CK(cudaGetLastError());
  return best;
}

// ---------------- MATCH.ANY.U64 ----------------
constexpr int ITERS = 4096;
__global__ void k_match(unsigned long long seed, unsigned* out) {
  unsigned lane = threadIdx.x & 31; unsigned acc = 0;
  unsigned long long key = (seed ^ (lane * 0x9E3779B97F4A7C15ull)) & 0xF;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    unsigned g = __match_any_sync(0xffffffffu, key);
    acc += g; key = (key + (g & 3)) & 0x1F;
  }
  if (acc == 0x12345) out[0] = acc;
}
__global__ void k_match32(unsigned seed, unsigned* out) {
  unsigned lane = threadIdx.x & 31; unsigned acc = 0;
  unsigned key = (seed ^ (lane * 0x9E3779B9u)) & 0xF;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    unsigned g = __match_any_sync(0xffffffffu, key);
    acc += g; key = (key + (g & 3)) & 0x1F;
  }
  if (acc == 0x12345) out[0] = acc;
}
__global__ void k_vote(unsigned seed, unsigned* out) {
  unsigned lane = threadIdx.x & 31; unsigned acc = 0; unsigned x = seed ^ lane;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    unsigned b = __ballot_sync(0xffffffffu, x & 1);
    acc += __popc(b); x = x * 1664525u + b;
  }
  if (acc == 0x12345) out[0] = acc;
}
struct GridArg { int blocks, threads; unsigned* out; };
static void l_match(void* p) { auto* a = (GridArg*)p; k_match<<<a->blocks, a->threads>>>(1, a->out); }
static void l_match32(void* p) { auto* a = (GridArg*)p; k_match32<<<a->blocks, a->threads>>>(1, a->out); }
static void l_vote(void* p) { auto* a = (GridArg*)p; k_vote<<<a->blocks, a->threads>>>(1, a->out); }

// ---------------- shared atomics ----------------
template <typename T>
__global__ void k_atoms(unsigned* out, int single_lane) {
  __shared__ T bins[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) bins[i] = 0;
  __syncthreads();
  unsigned x = threadIdx.x * 2654435761u + blockIdx.x;
  unsigned lane = threadIdx.x & 31;
#pragma unroll 4
  for (int i = 0; i < ITERS; ++i) {
    x = x * 1664525u + 1013904223u;
    if (!single_lane || lane == 0) atomicAdd(&bins[(x >> 8) & 4095], (T)1);
  }
  __syncthreads();
  if (threadIdx.x == 0 && bins[7] == (T)0x7fffffff) out[0] = 1;
}
static void l_atoms32(void* p) { auto* a = (GridArg*)p; k_atoms<unsigned><<<a->blocks, a->threads>>>(a->out, 0); }
static void l_atoms64(void* p) { auto* a = (GridArg*)p; k_atoms<unsigned long long><<<a->blocks, a->threads>>>(a->out, 0); }
static void l_atoms32_1(void* p) { auto* a = (GridArg*)p; k_atoms<unsigned><<<a->blocks, a->threads>>>(a->out, 1); }

// ---------------- global RED ----------------
__global__ void k_red(unsigned long long* dst, int nslots, int iters) {
  unsigned lane = threadIdx.x & 31;
  unsigned w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  for (int i = 0; i < iters; ++i)
    if (lane == 0) atomicAdd(&dst[((w + i * 7) % nslots) * 16], 1ull);
}
struct RedArg { int blocks, threads, nslots, iters; unsigned long long* dst; };
static void l_red(void* p) { auto* a = (RedArg*)p; k_red<<<a->blocks, a->threads>>>(a->dst, a->nslots, a->iters); }

// ---------------- HBM read ----------------
__global__ void k_read(const int4* __restrict__ src, size_t n, int4* sink) {
  int4 acc = make_int4(0, 0, 0, 0);
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    int4 v; asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + i));
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  if (acc.x == 0x7fffffff && acc.y == 3) sink[0] = acc;
}
struct ReadArg { int blocks, threads; const int4* src; size_t n; int4* sink; };
static void l_read(void* p) { auto* a = (ReadArg*)p; k_read<<<a->blocks, a->threads>>>(a->src, a->n, a->sink); }

// ---------------- stores into mapped pinned host memory ----------------
__global__ void k_hoststore16(int4* dst, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += stride)
    dst[i] = make_int4((int)i, 1, 2, 3);
}
__global__ void k_hoststore8(unsigned long long* dst, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += stride) dst[i] = i;
}
// one elected thread per CTA bulk-copies a 16 KB smem tile to the destination
__global__ void k_bulk(char* dst, size_t bytes) {
  extern __shared__ __align__(128) char tile[];
  const int TB = 16384;
  for (int i = threadIdx.x; i < TB / 16; i += blockDim.x) ((int4*)tile)[i] = make_int4(i, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    size_t ntiles = bytes / TB;
    for (size_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      unsigned saddr = (unsigned)__cvta_generic_to_shared(tile);
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                   :: "l"(dst + t * TB), "r"(saddr), "r"(TB) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 4;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}
struct HostArg { int blocks, threads; void* dst; size_t bytes; };
static void l_hs16(void* p) { auto* a = (HostArg*)p; k_hoststore16<<<a->blocks, a->threads>>>((int4*)a->dst, a->bytes / 16); }
static void l_hs8(void* p) { auto* a = (HostArg*)p; k_hoststore8<<<a->blocks, a->threads>>>((unsigned long long*)a->dst, a->bytes / 8); }
static void l_bulk(void* p) { auto* a = (HostArg*)p; k_bulk<<<a->blocks, 128, 16384>>>((char*)a->dst, a->bytes); }

int main() {
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0)); g_sms = prop.multiProcessorCount;
  int clk_khz = 0; CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0));
  unsigned* out; CK(cudaMalloc(&out, 64));
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"clock_attr_mhz\": %.0f", prop.name, g_sms, clk_khz / 1e3);
  // warp-op rates: report warp-ops per second chip-wide
  GridArg ga{g_sms * 8, 256, out};
  double warps = (double)ga.blocks * ga.threads / 32;
  float ms = time_kernel(l_match, &ga); printf(", \"match_u64_Gwarpop_s\": %.2f", warps * ITERS / (ms * 1e6));
  ms = time_kernel(l_match32, &ga); printf(", \"match_u32_Gwarpop_s\": %.2f", warps * ITERS / (ms * 1e6));
  ms = time_kernel(l_vote, &ga); printf(", \"vote_popc_Gwarpop_s\": %.2f", warps * ITERS / (ms * 1e6));
  ms = time_kernel(l_atoms32, &ga); printf(", \"atoms_u32_spread_Glane_s\": %.2f", warps * 32 * ITERS / (ms * 1e6));
  ms = time_kernel(l_atoms64, &ga); printf(", \"atoms_u64_spread_Glane_s\": %.2f", warps * 32 * ITERS / (ms * 1e6));
  ms = time_kernel(l_atoms32_1, &ga); printf(", \"atoms_u32_1lane_Gop_s\": %.2f", warps * ITERS / (ms * 1e6));
  // global RED
  unsigned long long* red; CK(cudaMalloc(&red, 16 * 8 * 65536)); CK(cudaMemset(red, 0, 16 * 8 * 65536));
  int slots[] = {1, 64, 65536};
  for (int s : slots) {
    RedArg ra{g_sms * 8, 256, s, 64, red};
    ms = time_kernel(l_red, &ra);
    printf(", \"red_u64_slots%d_Gop_s\": %.3f", s, (double)ra.blocks * 8 * ra.iters / (ms * 1e6));
  }
  // HBM read
  size_t bytes = (size_t)8 << 30; int4* src; CK(cudaMalloc(&src, bytes)); CK(cudaMemset(src, 1, bytes));
  int4* sink; CK(cudaMalloc(&sink, 64));
  for (int occ : {4, 8, 16}) {
    ReadArg rd{g_sms * occ, 256, src, bytes / 16, sink};
    ms = time_kernel(l_read, &rd);
    printf(", \"hbm_read_GBs_occ%d\": %.1f", occ, bytes / (ms * 1e6));
  }
  CK(cudaFree(src));
  // D2H
  size_t hb = (size_t)1 << 30; void* h; CK(cudaHostAlloc(&h, hb, cudaHostAllocMapped | cudaHostAllocPortable));
  void* hd; CK(cudaHostGetDevicePointer(&hd, h, 0));
  printf(", \"host_ptr_equals_dev_ptr\": %d", (int)(hd == h));
  void* dbuf; CK(cudaMalloc(&dbuf, hb));
  {
    cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    CK(cudaMemcpyAsync(h, dbuf, hb, cudaMemcpyDeviceToHost)); CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(a)); CK(cudaMemcpyAsync(h, dbuf, hb, cudaMemcpyDeviceToHost)); CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b)); CK(cudaEventElapsedTime(&ms, a, b));
    printf(", \"d2h_memcpy_GBs\": %.1f", hb / (ms * 1e6));
    CK(cudaEventRecord(a)); CK(cudaMemcpyAsync(dbuf, h, hb, cudaMemcpyHostToDevice)); CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b)); CK(cudaEventElapsedTime(&ms, a, b));
    printf(", \"h2d_memcpy_GBs\": %.1f", hb / (ms * 1e6));
  }
  for (int occ : {1, 4}) {
    HostArg ha{g_sms * occ, 256, hd, hb};
    ms = time_kernel(l_hs16, &ha, 3); printf(", \"sm_store16_host_GBs_occ%d\": %.1f", occ, hb / (ms * 1e6));
    ms = time_kernel(l_hs8, &ha, 3); printf(", \"sm_store8_host_GBs_occ%d\": %.1f", occ, hb / (ms * 1e6));
  }
  {
    HostArg ha{g_sms * 2, 128, hd, hb};
    ms = time_kernel(l_bulk, &ha, 3); printf(", \"bulk_copy_host_GBs\": %.1f", hb / (ms * 1e6));
    ms = time_kernel(l_hs16, &ha, 1);
    HostArg hd2{g_sms * 2, 128, dbuf, hb};
    ms = time_kernel(l_bulk, &hd2, 3); printf(", \"bulk_copy_hbm_GBs\": %.1f", hb / (ms * 1e6));
  }
  printf("}\n");
  return 0;
}
