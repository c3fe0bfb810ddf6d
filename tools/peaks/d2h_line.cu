// D2H protocol microbenchmark for the 128 B line transport (EM §5.2, C4 c4_line): each warp emits R records
// of one 128 B line (8 lanes x 16 B) into pinned, device-mapped host memory at 128 + 128 t, t a ticket, and
// commits them with a system-scope fence and 4 B tags in a dense tag array. Variants: tickets one per record
// (interleaved with other warps: the warp's tags land in scattered tag-array lines, one partial PCIe write
// each) or R at once (the warp's records and tags contiguous), with or without the commit. No consumer: the
// ring holds one pass. Prints records/s and GB/s of record bytes.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o d2h_line d2h_line.cu
#include <cstdio>
#include <cuda_runtime.h>

enum { PER_RECORD_TICKET = 1, COMMIT = 2 };

__global__ void k_emit(unsigned char* ring, unsigned* tags, unsigned long long* head, unsigned long long n_warp_blocks,
                       unsigned R, unsigned mode) {
  const unsigned lane = threadIdx.x & 31;
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  const unsigned long long w = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
  for (unsigned long long b = w; b < n_warp_blocks; b += warps) {
    unsigned long long t0 = 0;
    if (!(mode & PER_RECORD_TICKET)) {
      if (lane == 0) t0 = atomicAdd(head, (unsigned long long)R);
      t0 = __shfl_sync(0xffffffffu, t0, 0);
    }
    unsigned* tagp = nullptr;
    for (unsigned r = 0; r < R; ++r) {
      unsigned long long t = t0 + r;
      if (mode & PER_RECORD_TICKET) {
        if (lane == 0) t = atomicAdd(head, 1ull);
        t = __shfl_sync(0xffffffffu, t, 0);
      }
      unsigned char* rec = ring + 128 + t * 128;
      if (lane == r) tagp = tags + t;
      if (lane < 8) *reinterpret_cast<uint4*>(rec + 16 * lane) = make_uint4((unsigned)t, r, lane, 0u);
    }
    if (mode & COMMIT) {
      __threadfence_system();
      __syncwarp();
      if (lane < R) asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(tagp), "r"(1u) : "memory");
    }
  }
}

int main() {
  const size_t bytes = 1ull << 31;
  unsigned char* h = nullptr;
  cudaHostAlloc(&h, bytes + 4096, cudaHostAllocMapped);
  unsigned char* d = nullptr;
  cudaHostGetDevicePointer(&d, h, 0);
  unsigned* tags = nullptr;
  cudaHostAlloc(&tags, (bytes / 128 + 64) * 4, cudaHostAllocMapped);
  unsigned* dtags = nullptr;
  cudaHostGetDevicePointer(&dtags, tags, 0);
  unsigned long long* head = nullptr;
  cudaMalloc(&head, 8);
  struct Cfg { unsigned R, mode; const char* what; } cfgs[] = {
      {6, PER_RECORD_TICKET, "ticket per record, no commit"},
      {6, PER_RECORD_TICKET | COMMIT, "ticket per record, fence + 4 B tag per record (c4_line producer)"},
      {6, 0, "6 tickets per warp, no commit"},
      {6, COMMIT, "6 tickets per warp, fence + 6 contiguous tags"},
      {4, COMMIT, "4 tickets per warp, fence + 4 contiguous tags"},
      {8, COMMIT, "8 tickets per warp, fence + 8 contiguous tags"},
  };
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (auto& c : cfgs) {
    const unsigned long long recs = (bytes - 256) / 128;
    const unsigned long long blocks = recs / c.R;
    float best = 1e30f;
    for (int rep = 0; rep < 4; ++rep) {
      cudaMemset(head, 0, 8);
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0); cudaEventCreate(&e1);
      cudaEventRecord(e0);
      k_emit<<<sms * 3, 256>>>(d, dtags, head, blocks, c.R, c.mode);   // C4's 3 CTAs of 8 warps per SM
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      if (rep && ms < best) best = ms;
    }
    const double n = (double)blocks * c.R;
    printf("{\"what\": \"%s\", \"records_per_warp\": %u, \"record_GBs\": %.1f, \"Mrecords_s\": %.1f}\n", c.what, c.R,
           n * 128 / best / 1e6, n / best / 1e3);
  }
  return cudaGetLastError() != cudaSuccess;
}
