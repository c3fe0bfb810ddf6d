// Synthetic workloads with compiled-in injection points (C1-C4; EM §3.1-3.4) and their launchers.
//
// Each kernel is written once, in the "converged-hook discipline": lanes never return early; a lane
// that "exits" or is on the other side of a branch keeps running with in_flow = false, so every hook is
// reached by all 32 lanes and A/P are exact ballots (EM §1, reading R-15). Loops whose trip count
// varies per lane run warp-uniformly to the warp's maximum (SIMT-stack / IPDOM semantics). The
// template parameter T selects the instrumentation variant; T = 0 is the uninstrumented baseline.
#include <mutex>
#include <tuple>
#include <type_traits>

#include "nvbt_internal.h"
#include "nvbt_workloads.h"
#include "programs.cuh"
#include "workload_launch.cuh"

namespace nvbt {

template <class Prog> struct ProgTraits;

// ---------------------------------------------------------------- C1 vectorAdd (§3.1)
template <uint32_t T>
__global__ void __launch_bounds__(256) k_vectoradd(const float* __restrict__ a, const float* __restrict__ b,
                                                   float* __restrict__ c, int N, DevState st) {
  __shared__ __align__(16) unsigned sb[Hooks<T, ProgVectorAdd>::kSmemWords];
  Hooks<T, ProgVectorAdd> h(st, sb);
  const auto m0 = h.active(true);              // BB0: every lane
  const int tid = threadIdx.x;                 h.template at<0>(m0);
  const int cta = st.cta_lo + blockIdx.x;     h.template at<1>(m0);
  const int i = cta * 256 + tid;               h.template at<2>(m0);
  const bool p0 = i >= N;                      h.template at<3>(m0);
                                               h.template at<4>(m0, p0);  // @P0 EXIT
  const bool live = !p0;
  const auto m1 = h.active(live);              // BB1: lanes that did not exit
  const float* pa = a + i;                     h.template at<5>(m1);
  const float* pb = b + i;                     h.template at<6>(m1);
  float x = 0.f, y = 0.f;
  if (live) x = *pa;                           h.template at<7>(m1, true, (unsigned long long)pa);
  if (live) y = *pb;                           h.template at<8>(m1, true, (unsigned long long)pb);
  float* pc = c + i;                           h.template at<9>(m1);
  const float z = __fadd_rn(x, y);             h.template at<10>(m1);
  if (live) *pc = z;                           h.template at<11>(m1, true, (unsigned long long)pc);
                                               h.template at<12>(m1);
  h.finish();
}

// ---------------------------------------------------------------- C2 naive SGEMM (§3.2)
template <uint32_t T>
__global__ void __launch_bounds__(256, 6) k_sgemm(const float* __restrict__ A, const float* __restrict__ B,
                                               float* __restrict__ C, int M, int N, int K, DevState st) {
  __shared__ __align__(16) unsigned sb[Hooks<T, ProgSgemm>::kSmemWords];
  Hooks<T, ProgSgemm> h(st, sb);
  const auto m0 = h.active(true);
  const int tx = threadIdx.x;                  h.template at<0>(m0);
  const int ty = threadIdx.y;                  h.template at<1>(m0);
  const int bx = blockIdx.x;                   h.template at<2>(m0);
  const int by = st.cta_y0 + blockIdx.y;       h.template at<3>(m0);   // (partition: CTA-row offset)
  const int row = bx * 32 + tx;                h.template at<4>(m0);
  const int col = by * 8 + ty;                 h.template at<5>(m0);
  const bool p0 = row >= M || col >= N;        h.template at<6>(m0);
                                               h.template at<7>(m0, p0);  // @P0 EXIT
  const bool live = !p0;
  // BB1, every BB2 instance and BB3 have the same active mask (the lanes that did not exit): K is
  // warp-uniform, so the loop runs K times for every live lane.
  const auto m1 = h.active(live);
  float acc = 0.f;                             h.template at<8>(m1);
                                               h.template at<9>(m1);
  h.template retire<0, 9>();
  if (__any_sync(FULL, live)) {
    const float* pa = A + (size_t)row * K;
    const float* pb = B + col;
    auto instance = [&](int k) {               // BB2, instance k
      float x = 0.f, y = 0.f;
      if (live) x = pa[k];                     h.template at<10>(m1, true, (unsigned long long)(pa + k));
      if (live) y = pb[(size_t)k * N];         h.template at<11>(m1, true, (unsigned long long)(pb + (size_t)k * N));
      acc = fmaf(x, y, acc);                   h.template at<12>(m1);
                                               h.template at<13>(m1);
                                               h.template at<14>(m1);
                                               h.template at<15>(m1, k + 1 < K);  // @P1 BRA
    };
    constexpr int kChunk = (int)Hooks<T, ProgSgemm>::kSpillEvery;
    if (K <= kChunk) {                         // the u32 counters cannot wrap: the plain loop
      for (int k = 0; k < K; ++k) instance(k);
    } else {                                   // chunks of kChunk instances, counters spilled in between
      for (int k0 = 0; k0 < K; k0 += kChunk) {
        const int k1 = K - k0 > kChunk ? k0 + kChunk : K;
        for (int k = k0; k < k1; ++k) instance(k);
        if (k1 < K) h.spill();
      }
    }
  }
  float* pc = C + (size_t)row * N + col;
  if (live) *pc = acc;                         h.template at<16>(m1, true, (unsigned long long)pc);
                                               h.template at<17>(m1);
  h.finish();
}

// ---------------------------------------------------------------- C3 BFS (§3.3)
template <uint32_t T>
__global__ void __launch_bounds__(256) k_bfs_expand(const int* __restrict__ rowptr, const int* __restrict__ colidx,
                                                    int n, unsigned char* mask, const unsigned char* __restrict__ visited,
                                                    unsigned char* updating, DevState st) {
  __shared__ __align__(16) unsigned sb[Hooks<T, ProgBfs>::kSmemWords];
  Hooks<T, ProgBfs> h(st, sb);
  const auto m0 = h.active(true);
  const int tid = threadIdx.x;                 h.template at<0>(m0);
  const int cta = st.cta_lo + blockIdx.x;     h.template at<1>(m0);
  const int t = cta * 256 + tid;               h.template at<2>(m0);
  const bool p0 = t >= n;                      h.template at<3>(m0);
                                               h.template at<4>(m0, p0);  // @P0 EXIT
  const bool live = !p0;
  const auto m1 = h.active(live);              // BB1 (and BB6 after reconvergence)
  unsigned char mk = 0;
  if (live) mk = mask[t];                      h.template at<5>(m1, true, (unsigned long long)(mask + t));
  const bool p1 = mk != 0;                     h.template at<6>(m1);
                                               h.template at<7>(m1, !p1);  // @!P1 BRA exit
  const bool front = live && p1;
  h.template retire<0, 7>();
  const auto m2 = h.active(front);             // BB2: frontier lanes
  int start = 0, end = 0;
  if (front) mask[t] = 0;                      h.template at<8>(m2, true, (unsigned long long)(mask + t));
  if (front) start = rowptr[t];                h.template at<9>(m2, true, (unsigned long long)(rowptr + t));
  if (front) end = rowptr[t + 1];              h.template at<10>(m2, true, (unsigned long long)(rowptr + t + 1));
  const bool p2 = start >= end;                h.template at<11>(m2);
                                               h.template at<12>(m2, p2);  // @P2 BRA exit
  h.template retire<8, 12>();
  bool in_loop = front && !p2;
  int e = start;
  auto instance = [&]() {                      // warp-uniform edge loop; instance k has e = start + k
    const auto m3 = h.active(in_loop);         // BB3 and BB5 of this instance
    int nb = 0;
    if (in_loop) nb = colidx[e];               h.template at<13>(m3, true, (unsigned long long)(colidx + e));
    unsigned char v = 0;
    if (in_loop) v = visited[nb];              h.template at<14>(m3, true, (unsigned long long)(visited + nb));
    const bool p3 = v != 0;                    h.template at<15>(m3);
                                               h.template at<16>(m3, p3);  // @P3 BRA
    const bool unv = in_loop && !p3;
    const auto m4 = h.active(unv);             // BB4: unvisited neighbour
    if (unv) updating[nb] = 1;                 h.template at<17>(m4, true, (unsigned long long)(updating + nb));
    const int e1 = e + 1;                      h.template at<18>(m3);
    const bool p4 = e1 < end;                  h.template at<19>(m3);
                                               h.template at<20>(m3, p4);  // @P4 BRA loop
    if (in_loop) e = e1;
    in_loop = in_loop && p4;
  };
  // exact while every warp's trip count (its largest degree) is < 2^24: the register counters grow by
  // <= 32 and the per-warp totals by <= 8 x 32 per instance into u32 CTA bins. A larger hub (which a
  // chunked loop with spills could handle, but whose code raises the plain loop's registers 28 -> 40
  // and costs the latency-bound BFS occupancy) is flagged: the read calls then return NVBT_EINVAL.
  if constexpr (Hooks<T, ProgBfs>::kOn) {
    if (__any_sync(FULL, in_loop && end - start >= (1 << 24)) && (threadIdx.x & 31u) == 0u) atomicAdd(st.ovf, 1ull);
  }
  while (__any_sync(FULL, in_loop)) instance();
                                               h.template at<21>(m1);
  h.finish();
}

template <uint32_t T>
__global__ void __launch_bounds__(256) k_bfs_update(int n, unsigned char* mask, unsigned char* visited,
                                                    unsigned char* updating, int* cost, int* over, int level,
                                                    DevState st) {
  __shared__ __align__(16) unsigned sb[Hooks<T, ProgBfs>::kSmemWords];
  Hooks<T, ProgBfs> h(st, sb);
  const auto m0 = h.active(true);
  const int tid = threadIdx.x;                 h.template at<22>(m0);
  const int cta = st.cta_lo + blockIdx.x;     h.template at<23>(m0);
  const int t = cta * 256 + tid;               h.template at<24>(m0);
  const bool p0 = t >= n;                      h.template at<25>(m0);
                                               h.template at<26>(m0, p0);
  const bool live = !p0;
  const auto m1 = h.active(live);              // BB8 (and BB10)
  unsigned char u = 0;
  if (live) u = updating[t];                   h.template at<27>(m1, true, (unsigned long long)(updating + t));
  const bool p1 = u != 0;                      h.template at<28>(m1);
                                               h.template at<29>(m1, !p1);
  const bool up = live && p1;
  const auto m2 = h.active(up);                // BB9
  if (up) mask[t] = 1;                         h.template at<30>(m2, true, (unsigned long long)(mask + t));
  if (up) visited[t] = 1;                      h.template at<31>(m2, true, (unsigned long long)(visited + t));
  if (up) cost[t] = level + 1;                 h.template at<32>(m2, true, (unsigned long long)(cost + t));
  if (up) updating[t] = 0;                     h.template at<33>(m2, true, (unsigned long long)(updating + t));
  if (up) *over = 1;                           h.template at<34>(m2, true, (unsigned long long)over);
                                               h.template at<35>(m1);
  h.finish();
}

// ---------------------------------------------------------------- C4 5-point stencil (§3.4)
template <uint32_t T>
__global__ void __launch_bounds__(256) k_stencil(const float* __restrict__ in, float* __restrict__ out, int n,
                                                 DevState st) {
  __shared__ __align__(16) unsigned sb[Hooks<T, ProgStencil>::kSmemWords];
  Hooks<T, ProgStencil> h(st, sb);
  const auto m0 = h.active(true);
  const int tx = threadIdx.x;                  h.template at<0>(m0);
  const int ty = threadIdx.y;                  h.template at<1>(m0);
  const int bx = blockIdx.x;                   h.template at<2>(m0);
  const int by = st.cta_y0 + blockIdx.y;       h.template at<3>(m0);   // (partition: CTA-row offset)
  const int j = bx * 32 + tx;                  h.template at<4>(m0);
  const int i = by * 8 + ty;                   h.template at<5>(m0);
  const bool p0 = i >= n || j >= n;            h.template at<6>(m0);
                                               h.template at<7>(m0, p0);
  const bool live = !p0;
  const auto m1 = h.active(live);              // BB1 (boundaries are predicated, not branched)
  const bool p1 = live && i > 0 && i < n - 1 && j > 0 && j < n - 1;
                                               h.template at<8>(m1);
  const size_t o = (size_t)i * n + j;
  float c = 0.f, u = 0.f, d = 0.f, l = 0.f, r = 0.f;
  if (live) c = in[o];                         h.template at<9>(m1, true, (unsigned long long)(in + o));
  if (p1) u = in[o - n];                       h.template at<10>(m1, p1, (unsigned long long)(in + o - n));
  if (p1) d = in[o + n];                       h.template at<11>(m1, p1, (unsigned long long)(in + o + n));
  if (p1) l = in[o - 1];                       h.template at<12>(m1, p1, (unsigned long long)(in + o - 1));
  if (p1) r = in[o + 1];                       h.template at<13>(m1, p1, (unsigned long long)(in + o + 1));
  float s = __fadd_rn(u, d);                   h.template at<14>(m1, p1);
  s = __fadd_rn(s, l);                         h.template at<15>(m1, p1);
  s = __fadd_rn(s, r);                         h.template at<16>(m1, p1);
  s = __fmul_rn(0.25f, s);                     h.template at<17>(m1, p1);
  const float v = p1 ? s : c;                  h.template at<18>(m1);
  if (live) out[o] = v;                        h.template at<19>(m1, true, (unsigned long long)(out + o));
                                               h.template at<20>(m1);
  h.finish();
}

}  // namespace nvbt

using namespace nvbt;

// Dynamic shared memory that caps k_stencil<T> (256 threads) at 3 CTAs per SM on `dev`: 4 x (dyn + static
// + per-block reserved) must exceed the SM's shared memory, 3 x must fit. Derived from the kernel's own
// static size and the device's limits, checked with the occupancy calculator, cached per (kernel, device).
// Dynamic shared memory that caps a host-channel traced stencil at kC CTAs per SM (see nvbt_stencil).
static int stencil_pad(const void* fn, int dev, int kC, size_t* dyn) {
  static std::mutex m;
  static std::vector<std::tuple<const void*, int, size_t, int>> cache;
  {
    std::lock_guard<std::mutex> g(m);
    for (auto& c : cache)
      if (std::get<0>(c) == fn && std::get<1>(c) == dev && std::get<3>(c) == kC) { *dyn = std::get<2>(c); return NVBT_OK; }
  }
  cudaFuncAttributes fa{};
  int per_sm = 0, reserved = 0;
  NVBT_CUDA(cudaFuncGetAttributes(&fa, fn));
  NVBT_CUDA(cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  NVBT_CUDA(cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev));
  const size_t used = fa.sharedSizeBytes + (size_t)reserved;
  const size_t part = (size_t)per_sm / (kC + 1) + 128;        // kC + 1 CTAs of this size exceed the SM
  const size_t d = part > used ? ((part - used + 127) & ~size_t(127)) : 0;
  if (kC * (d + used) > (size_t)per_sm) return set_error(NVBT_ECUDA, "stencil pad: %d CTAs do not fit (%zu B)", kC, d);
  int rc = func_smem(fn, dev, d);
  if (rc) return rc;
  int blocks = 0;
  NVBT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, fn, 256, d));
  if (blocks > kC || blocks < 1)
    return set_error(NVBT_ECUDA, "stencil pad %zu B gives %d CTAs per SM, expected <= %d", d, blocks, kC);
  std::lock_guard<std::mutex> g(m);
  cache.emplace_back(fn, dev, d, kC);
  *dyn = d;
  return NVBT_OK;
}

extern "C" {

int nvbt_program(int w, nvbt_instr_desc* out, uint32_t cap, uint32_t* n_pcs, uint32_t* n_ops, uint32_t* n_bbs);

int nvbt_workload_warps(int w, const int64_t* a, uint32_t na, uint64_t* n) {
  if (!a || !n) return set_error(NVBT_EINVAL, "null argument");
  switch (w) {
    case NVBT_W_VECTORADD: case NVBT_W_BFS:
      if (na < 1 || a[0] < 0) break;
      *n = (uint64_t)((a[0] + 255) / 256) * 8; return NVBT_OK;
    case NVBT_W_SGEMM:
      if (na < 2 || a[0] < 0 || a[1] < 0) break;
      *n = (uint64_t)((a[0] + 31) / 32) * (uint64_t)((a[1] + 7) / 8) * 8; return NVBT_OK;
    case NVBT_W_STENCIL:
      if (na < 1 || a[0] < 0) break;
      *n = (uint64_t)((a[0] + 31) / 32) * (uint64_t)((a[0] + 7) / 8) * 8; return NVBT_OK;
    case NVBT_W_WFFT_EMU: case NVBT_W_WFFT_SW:
      if (na < 2 || a[0] < 0 || a[1] < 1) break;
      *n = (uint64_t)a[1] * 8; return NVBT_OK;
    default: break;
  }
  return set_error(NVBT_EINVAL, "bad workload %d or arguments", w);
}

}  // extern "C"

namespace nvbt {
int preload_workload_kernels(int dev) {
  static std::mutex mu;
  static bool done_dev[64] = {};
  std::lock_guard<std::mutex> g(mu);
  if (dev < 0 || dev >= 64 || done_dev[dev]) return NVBT_OK;
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  auto load = [&](const void* fn) { if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, fn); };
  for (uint32_t t : {0u, 1u, 2u, 4u, 5u, 6u, 8u, 9u, 10u, 12u, 13u, 14u}) {
    dispatch(t, [&](auto tag) {
      constexpr uint32_t T = decltype(tag)::value;
      load((const void*)k_vectoradd<T>);
      load((const void*)k_sgemm<T>);
    });
    for (bool dev_ring : {false, true})
      dispatch_trace(t, dev_ring, [&](auto tag) {
        constexpr uint32_t T = decltype(tag)::value;
        load((const void*)k_bfs_expand<T>);
        load((const void*)k_bfs_update<T>);
        load((const void*)k_stencil<T>);
      });
  }
  if (e != cudaSuccess) return set_error(NVBT_ECUDA, "kernel preload: %s", cudaGetErrorString(e));
  done_dev[dev] = true;
  return NVBT_OK;
}
}  // namespace nvbt

extern "C" {

int nvbt_vectoradd(nvbt_ctx ctx, void* stream, uint32_t tools, const float* a, const float* b, float* c, int32_t N) {
  if (!a || !b || !c || N < 0) return set_error(NVBT_EINVAL, "bad vectorAdd arguments");
  LaunchCtx lc;
  int rc = prepare<ProgVectorAdd>(ctx, stream, tools, "vectorAdd", &lc);
  if (!rc) rc = partition(ctx, 1, (N + 255) / 256, &lc);
  if (rc) return rc;
  if (lc.n_ctas == 0) return NVBT_OK;
  rc = dispatch(tools, [&](auto tag) { k_vectoradd<decltype(tag)::value><<<lc.grid, 256, 0, lc.stream>>>(a, b, c, N, lc.st); });
  return rc ? rc : done(ctx, 1);
}

int nvbt_sgemm(nvbt_ctx ctx, void* stream, uint32_t tools, const float* A, const float* B, float* C, int32_t M,
               int32_t N, int32_t K) {
  if (!A || !B || !C || M < 0 || N < 0 || K < 1) return set_error(NVBT_EINVAL, "bad SGEMM arguments");
  LaunchCtx lc;
  int rc = prepare<ProgSgemm>(ctx, stream, tools, "SGEMM", &lc);
  if (!rc) rc = partition(ctx, (M + 31) / 32, (N + 7) / 8, &lc);
  if (rc) return rc;
  if (lc.n_ctas == 0) return NVBT_OK;
  const dim3 block(32, 8);
  rc = dispatch(tools, [&](auto tag) { k_sgemm<decltype(tag)::value><<<lc.grid, block, 0, lc.stream>>>(A, B, C, M, N, K, lc.st); });
  return rc ? rc : done(ctx, 1);
}

// C3 kernels 1 and 2 as separate launches (a multi-GPU BFS exchanges `updating` between them).
static int bfs_launch(nvbt_ctx ctx, void* stream, uint32_t tools, int which, const int32_t* rowptr, const int32_t* col,
                      int32_t n, uint8_t* mask, uint8_t* visited, uint8_t* updating, int32_t* cost, int32_t* over,
                      int32_t level) {
  if (!mask || !visited || !updating || n < 0 || (which != 2 && (!rowptr || !col)) || (which != 1 && (!cost || !over)))
    return set_error(NVBT_EINVAL, "bad BFS arguments");
  LaunchCtx l1, l2;
  int rc = NVBT_OK;
  if (which & 1) {
    rc = prepare<ProgBfs>(ctx, stream, tools, "BFS", &l1);
    if (!rc) rc = partition(ctx, 1, (n + 255) / 256, &l1);
  }
  if (!rc && (which & 2)) {   // kernel 2 is a launch of its own (next launch id)
    rc = prepare<ProgBfs>(ctx, stream, tools, "BFS", &l2);
    if (!rc) rc = partition(ctx, 1, (n + 255) / 256, &l2);
  }
  if (rc) return rc;
  const unsigned nc = (which & 1) ? l1.n_ctas : l2.n_ctas;
  if (nc == 0) return NVBT_OK;
  rc = dispatch_trace(tools, ((which & 1) ? l1.st : l2.st).no_wait != 0u, [&](auto tag) {
    constexpr uint32_t TT = decltype(tag)::value;
    if (which & 1) k_bfs_expand<TT><<<l1.grid, 256, 0, l1.stream>>>(rowptr, col, n, mask, visited, updating, l1.st);
    if (which & 2) k_bfs_update<TT><<<l2.grid, 256, 0, l2.stream>>>(n, mask, visited, updating, cost, over, level, l2.st);
  });
  return rc ? rc : done(ctx, which == 3 ? 2 : 1);
}

int nvbt_bfs_level(nvbt_ctx ctx, void* stream, uint32_t tools, const int32_t* rowptr, const int32_t* col, int32_t n,
                   uint8_t* mask, uint8_t* visited, uint8_t* updating, int32_t* cost, int32_t* over, int32_t level) {
  if (!rowptr || !col || !cost || !over) return set_error(NVBT_EINVAL, "bad BFS arguments");
  return bfs_launch(ctx, stream, tools, 3, rowptr, col, n, mask, visited, updating, cost, over, level);
}

int nvbt_bfs_expand(nvbt_ctx ctx, void* stream, uint32_t tools, const int32_t* rowptr, const int32_t* col, int32_t n,
                    uint8_t* mask, const uint8_t* visited, uint8_t* updating) {
  return bfs_launch(ctx, stream, tools, 1, rowptr, col, n, mask, const_cast<uint8_t*>(visited), updating, nullptr,
                    nullptr, 0);
}

int nvbt_bfs_update(nvbt_ctx ctx, void* stream, uint32_t tools, int32_t n, uint8_t* mask, uint8_t* visited,
                    uint8_t* updating, int32_t* cost, int32_t* over, int32_t level) {
  return bfs_launch(ctx, stream, tools, 2, nullptr, nullptr, n, mask, visited, updating, cost, over, level);
}

int nvbt_stencil(nvbt_ctx ctx, void* stream, uint32_t tools, const float* in, float* out, int32_t n) {
  if (!in || !out || n < 0) return set_error(NVBT_EINVAL, "bad stencil arguments");
  LaunchCtx lc;
  int rc = prepare<ProgStencil>(ctx, stream, tools, "stencil", &lc);
  if (!rc) rc = partition(ctx, (n + 31) / 32, (n + 7) / 8, &lc);
  if (rc) return rc;
  if (lc.n_ctas == 0) return NVBT_OK;
  const dim3 block(32, 8);
  int pad_rc = NVBT_OK;
  rc = dispatch_trace(tools, lc.st.no_wait != 0u, [&](auto tag) {
    constexpr uint32_t T = decltype(tag)::value;
    size_t dyn = 0;
    if constexpr ((T & TOOL_TRACE) && !(T & TOOL_TRACE_DEV)) {
      // Host-channel producer: at most 3 CTAs (24 warps) per SM, 6 for 128 B line slots, enforced by padding
      // dynamic shared memory just past 1/4 (1/7) of the SM's shared memory. The PCIe link is saturated;
      // fewer warps fencing at once move more records (round 1, per-record tickets: uncapped 147 M
      // records/s, 3 CTAs 151, 2 CTAs 154; round 2, staged blocks (profiles/r2_c4_ctas_ab.txt): 288 B
      // 2 / 3 / 4 / 6 CTAs 149 / 161 / 162 / 161 M, 176 B 226 / 242 / 242 / 238 M, 128 B lines 313 / 325-332 /
      // 326 / 345 M).
      pad_rc = stencil_pad((const void*)k_stencil<T>, ctx->device, lc.st.compact >= 3u ? 6 : 3, &dyn);
      if (pad_rc) return;
    }
    k_stencil<T><<<lc.grid, block, dyn, lc.stream>>>(in, out, n, lc.st);
  });
  if (pad_rc) return pad_rc;
  return rc ? rc : done(ctx, 1);
}

int nvbt_set_partition(nvbt_ctx ctx, uint32_t rank, uint32_t world) {
  if (!ctx || world == 0 || rank >= world) return set_error(NVBT_EINVAL, "bad partition rank %u of %u", rank, world);
  ctx->part_rank = rank;
  ctx->part_world = world;
  return NVBT_OK;
}

}  // extern "C"
