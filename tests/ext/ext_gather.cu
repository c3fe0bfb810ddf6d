// An instrumented kernel OUTSIDE libnvbt.so, written against the public device API only
// (include/nvbt_dev.cuh + include/nvbt.h): the test of SURVEY §8(b)'s device hook header. It is the
// compiled-in analogue of an NVBit tool instrumenting someone else's kernel (nvbit_insert_call at each
// instruction of interest, P:L123 (§4)): a data-dependent gather y[i] = 2 x[idx[i]] + 1, read only when
// idx[i] % 3 != 0. Its program table (tests/test_gpu_device_api.py PROGRAM):
//   pc0 S2R | pc1 ISETP | pc2 @P0 EXIT, P0 = i >= n            (bb0: leader pc0; pc2 guarded)
//   pc3 LDG idx[i] | pc4 @P1 LDG x[idx[i]], P1 = idx[i] % 3 != 0 | pc5 FFMA | pc6 STG y[i] | pc7 EXIT
//                                                              (bb1: leader pc3; pc4 guarded)
// Hooks follow the tools the context handed out: COUNT (every pc), BBCOUNT (block leaders + guarded pcs),
// MEMDIV (the three global LD/ST pcs).
#include <cuda_runtime.h>
#include "nvbt_dev.cuh"

__global__ void ext_gather(nvbt_dev_state st, const int* idx, const float* x, float* y, int n) {
  extern __shared__ __align__(16) unsigned char smem[];
  nvbt_hooks h;
  nvbt_cta_begin(h, st, smem);
  const bool cnt = (st.tools & NVBT_TOOL_COUNT) != 0, bb = (st.tools & NVBT_TOOL_BBCOUNT) != 0;
  const bool mem = (st.tools & NVBT_TOOL_MEMDIV) != 0;
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  // bb0
  if (bb) nvbt_on_bb(h, 0, true, 3);
  if (cnt) {
    nvbt_on_instr(h, 0, true);
    nvbt_on_instr(h, 1, true);
  }
  if (cnt || bb) nvbt_on_instr(h, 2, true, i >= n);
  const bool live = i < n;                        // lanes that executed the EXIT are gone
  // bb1
  const int k = live ? idx[i] : 0;
  const bool p1 = live && (k % 3) != 0;
  if (bb) nvbt_on_bb(h, 3, live, 5);
  if (cnt) nvbt_on_instr(h, 3, live);
  if (mem) nvbt_on_mem(h, 3, live, true, (uint64_t)(idx + i));
  if (cnt || bb) nvbt_on_instr(h, 4, live, p1);
  if (mem) nvbt_on_mem(h, 4, live, p1, (uint64_t)(x + k));
  const float v = p1 ? x[k] : 0.f;
  if (cnt) {
    nvbt_on_instr(h, 5, live);
    nvbt_on_instr(h, 6, live);
  }
  if (mem) nvbt_on_mem(h, 6, live, true, (uint64_t)(y + i));
  if (live) y[i] = 2.f * v + 1.f;
  if (cnt) nvbt_on_instr(h, 7, live);
  nvbt_cta_flush(h);
}

extern "C" int ext_gather_launch(const nvbt_dev_state* st, const int* idx, const float* x, float* y, int n,
                                 int block, void* stream) {
  if (n <= 0) return 0;
  const size_t smem = NVBT_DEV_SMEM_BYTES(st->n_pcs, block / 32);
  ext_gather<<<(n + block - 1) / block, block, smem, static_cast<cudaStream_t>(stream)>>>(*st, idx, x, y, n);
  return (int)cudaGetLastError();
}
