// D2H write-pattern microbenchmark (C4 transport analysis): warps write fixed-size records into pinned,
// device-mapped host memory with 16 B per-lane stores, record r by warp (r mod warps), records packed at a
// given stride. Prints GB/s of record bytes for several record sizes / strides / alignments.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o d2h_pattern d2h_pattern.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_write(unsigned char* ring, unsigned long long n_rec, unsigned rec_bytes, unsigned stride,
                        unsigned offset) {
  const unsigned lane = threadIdx.x & 31;
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  const unsigned long long w = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
  const unsigned chunks = rec_bytes / 16;
  for (unsigned long long r = w; r < n_rec; r += warps) {
    unsigned char* rec = ring + offset + r * stride;
    for (unsigned c = lane; c < chunks; c += 32)
      *reinterpret_cast<uint4*>(rec + 16 * c) = make_uint4((unsigned)r, c, 1u, 2u);
  }
}

int main() {
  const size_t bytes = 1ull << 31;
  unsigned char* h = nullptr;
  cudaHostAlloc(&h, bytes + 4096, cudaHostAllocMapped);
  unsigned char* d = nullptr;
  cudaHostGetDevicePointer(&d, h, 0);
  struct Cfg { unsigned rec, stride, offset; const char* what; } cfgs[] = {
      {256, 256, 0, "256 B records, 256 B stride (line aligned)"},
      {288, 288, 64, "288 B records, 288 B stride, ring data at +64 (the C4 ring)"},
      {288, 288, 0, "288 B records, 288 B stride, ring data at +0"},
      {288, 384, 0, "288 B records in 384 B slots (3 lines each)"},
      {1152, 1152, 0, "1152 B blocks (4 x 288 B, 9 full lines)"},
      {176, 176, 64, "176 B compact slots at +64"},
      {176, 176, 0, "176 B compact slots at +0"},
      {176, 192, 0, "176 B compact records in 192 B slots at +0"},
      {176, 192, 64, "176 B compact records in 192 B slots at +64"},
      {176, 192, 128, "176 B compact records in 192 B slots at +128"},
      {176, 256, 0, "176 B compact records in 256 B slots at +0"},
      {128, 128, 0, "128 B records, 128 B stride (one line each)"},
      {288, 320, 0, "288 B records in 320 B slots at +0 (pairs of slots = 5 lines)"},
      {288, 320, 64, "288 B records in 320 B slots at +64"},
      {256, 256, 64, "256 B records, 256 B stride at +64"},
  };
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (const Cfg& c : cfgs) {
    const unsigned long long n = (bytes - c.offset) / c.stride;
    float best = 1e30f;
    for (int it = 0; it < 4; ++it) {
      cudaEventRecord(e0);
      k_write<<<sms * 8, 256>>>(d, n, c.rec, c.stride, c.offset);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (it > 0 && ms < best) best = ms;
    }
    printf("{\"what\": \"%s\", \"record_GBs\": %.1f, \"link_bytes_GBs\": %.1f}\n", c.what,
           n * (double)c.rec / (best * 1e-3) / 1e9, n * (double)c.stride / (best * 1e-3) / 1e9);
  }
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
  return 0;
}
