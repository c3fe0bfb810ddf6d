// D2H channel-protocol microbenchmark (C4 transport analysis, DESIGN §9 item 4): the C4 producer's
// protocol without the stencil around it. Each warp emits R records of 288 B (18 lanes x 16 B) into pinned,
// device-mapped host memory at 64 + 288 t, t a ticket from one global counter, then commits: a system-scope
// fence and one 4 B tag store per record (byte 28). Variants separate the costs: tickets taken one per
// record (interleaved with other warps, as the C4 producer does) or R at once (a warp's records
// contiguous), with or without the commit, and one tag per block instead of per record.
// No host consumer: the ring is large enough for one pass. Prints GB/s of record bytes.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o d2h_protocol d2h_protocol.cu
#include <cstdio>
#include <cuda_runtime.h>

enum { PER_RECORD_TICKET = 1, COMMIT = 2, BLOCK_TAG = 4, TAG_ARRAY = 8, NO_FENCE = 16, DATA_AT_128 = 32 };

__global__ void k_emit(unsigned char* ring, unsigned* tags, unsigned long long* head, unsigned long long n_warp_blocks, unsigned R,
                       unsigned mode) {
  const unsigned lane = threadIdx.x & 31;
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  const unsigned long long w = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
  for (unsigned long long b = w; b < n_warp_blocks; b += warps) {
    unsigned long long t0 = 0;
    if (!(mode & PER_RECORD_TICKET)) {
      if (lane == 0) t0 = atomicAdd(head, (unsigned long long)R);
      t0 = __shfl_sync(0xffffffffu, t0, 0);
    }
    unsigned char* tagp = nullptr;
    for (unsigned r = 0; r < R; ++r) {
      unsigned long long t = t0 + r;
      if (mode & PER_RECORD_TICKET) {
        if (lane == 0) t = atomicAdd(head, 1ull);
        t = __shfl_sync(0xffffffffu, t, 0);
      }
      unsigned char* rec = ring + ((mode & DATA_AT_128) ? 128 : 64) + t * 288;
      if (lane == r) tagp = (mode & TAG_ARRAY) ? reinterpret_cast<unsigned char*>(tags + t) : rec + 28;
      if (lane < 18) *reinterpret_cast<uint4*>(rec + 16 * lane) = make_uint4((unsigned)t, r, lane, 0u);
    }
    if (mode & COMMIT) {
      if (!(mode & NO_FENCE)) __threadfence_system();
      __syncwarp();
      const unsigned ntag = (mode & BLOCK_TAG) ? 1u : R;
      if (lane < ntag) asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(tagp), "r"(1u) : "memory");
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
  cudaHostAlloc(&tags, (bytes / 288 + 64) * 4, cudaHostAllocMapped);
  unsigned* dtags = nullptr;
  cudaHostGetDevicePointer(&dtags, tags, 0);
  unsigned long long* head = nullptr;
  cudaMalloc(&head, 8);
  struct Cfg { unsigned R, mode; const char* what; } cfgs[] = {
      {6, PER_RECORD_TICKET, "ticket per record, no commit"},
      {6, PER_RECORD_TICKET | COMMIT, "ticket per record, fence + 4 B tag per record (C4 producer)"},
      {6, 0, "6 tickets per warp, no commit"},
      {6, COMMIT, "6 tickets per warp, fence + 4 B tag per record"},
      {6, COMMIT | BLOCK_TAG, "6 tickets per warp, fence + one 4 B tag per block"},
      {4, 0, "4 tickets per warp, no commit"},
      {4, COMMIT | BLOCK_TAG, "4 tickets per warp, fence + one 4 B tag per block"},
      {6, PER_RECORD_TICKET | COMMIT | NO_FENCE, "ticket per record, 4 B tag per record, no fence"},
      {6, PER_RECORD_TICKET | COMMIT | TAG_ARRAY, "ticket per record, fence + 4 B tag per record in a dense tag array"},
      {6, PER_RECORD_TICKET | COMMIT | TAG_ARRAY | NO_FENCE, "ticket per record, 4 B tag per record in a dense tag array, no fence"},
      {6, COMMIT | TAG_ARRAY, "6 tickets per warp, fence + 6 tags (24 B) in a dense tag array"},
      {4, COMMIT | TAG_ARRAY | DATA_AT_128, "4 tickets per warp, data at +128, fence + 4 tags in a dense tag array"},
      {4, DATA_AT_128, "4 tickets per warp, data at +128, no commit"},
  };
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (const Cfg& c : cfgs) {
    const unsigned long long n_rec = (bytes - 64) / 288, nb = n_rec / c.R;
    float best = 1e30f;
    for (int it = 0; it < 4; ++it) {
      cudaMemset(head, 0, 8);
      cudaEventRecord(e0);
      k_emit<<<sms * 8, 256>>>(d, dtags, head, nb, c.R, c.mode);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (it > 0 && ms < best) best = ms;
    }
    printf("{\"what\": \"%s\", \"records_per_warp\": %u, \"record_GBs\": %.1f, \"Mrecords_s\": %.1f}\n", c.what,
           c.R, nb * c.R * 288.0 / (best * 1e-3) / 1e9, nb * c.R / (best * 1e-3) / 1e6);
  }
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
