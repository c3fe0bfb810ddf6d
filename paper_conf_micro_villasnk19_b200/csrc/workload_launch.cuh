// Launch helpers shared by the workload translation units (workloads.cu, wfft.cu).
#pragma once
#include <type_traits>

#include "nvbt_internal.h"

namespace nvbt {

// ---------------------------------------------------------------- dispatch over tool variants
template <class F>
static inline int dispatch(uint32_t tools, F&& f) {
#define NVBT_CASE(v) case v: f(std::integral_constant<uint32_t, v>{}); return NVBT_OK;
  switch (tools) {
    NVBT_CASE(0) NVBT_CASE(1) NVBT_CASE(2) NVBT_CASE(4) NVBT_CASE(5) NVBT_CASE(6) NVBT_CASE(8) NVBT_CASE(9)
    NVBT_CASE(10) NVBT_CASE(12) NVBT_CASE(13) NVBT_CASE(14)
    default: return set_error(NVBT_EINVAL, "unsupported tools combination 0x%x", tools);
  }
#undef NVBT_CASE
}

// Workloads that trace into device rings (F2: stencil, BFS) also have TRACE variants with the device-ring
// producer selected at compile time (TOOL_TRACE_DEV); other contexts take the run-time channel path.
template <class F>
static inline int dispatch_trace(uint32_t tools, bool dev_ring, F&& f) {
  if ((tools & NVBT_TOOL_TRACE) != 0 && dev_ring) {
#define NVBT_CASE(v) case v: f(std::integral_constant<uint32_t, v | TOOL_TRACE_DEV>{}); return NVBT_OK;
    switch (tools) {
      NVBT_CASE(8) NVBT_CASE(9) NVBT_CASE(10) NVBT_CASE(12) NVBT_CASE(13) NVBT_CASE(14)
      default: return set_error(NVBT_EINVAL, "unsupported tools combination 0x%x", tools);
    }
#undef NVBT_CASE
  }
  return dispatch(tools, f);
}

struct LaunchCtx {
  cudaStream_t stream = nullptr;
  DevState st{};
  dim3 grid{0, 1, 1};    // the launch's share of the CTA grid
  unsigned n_ctas = 0;
};

// Multi-GPU partition (nvbt_set_partition): a workload whose CTA grid has gy rows of gx
// CTAs (1D grids: gx = 1) runs, on rank r of w, the whole CTA rows [gy r / w, gy (r + 1) / w), i.e. the
// logical CTAs [gx gy r / w, ...) in linear order: 2D workloads launch (gx, rows) with ctaid.y offset by
// cta_y0, 1D workloads launch (rows) with the CTA id offset by cta_lo. Global warp ids, addresses and hence
// every event are those of the unpartitioned launch, so per-rank results sum to the full result.
// Must follow prepare() (which rebuilds lc->st).
static inline int partition(nvbt_ctx ctx, unsigned long long gx, unsigned long long gy, LaunchCtx* lc) {
  const unsigned long long r = ctx ? ctx->part_rank : 0, w = ctx ? ctx->part_world : 1;
  const unsigned long long y0 = gy * r / w, y1 = gy * (r + 1) / w;
  if (gx * gy > 0x7fffffffull || (gx > 1 && gy > 65535)) return set_error(NVBT_EINVAL, "CTA grid too large");
  lc->st.cta_lo = (unsigned)(gx * y0);
  lc->st.cta_y0 = (unsigned)y0;
  lc->n_ctas = (unsigned)(gx * (y1 - y0));
  lc->grid = gx > 1 ? dim3((unsigned)gx, (unsigned)(y1 - y0), 1) : dim3((unsigned)(y1 - y0), 1, 1);
  return NVBT_OK;
}

template <class Prog>
static inline int prepare(nvbt_ctx ctx, void* stream, uint32_t tools, const char* name, LaunchCtx* lc) {
  if (tools != 0) {
    if (!ctx) return set_error(NVBT_EINVAL, "instrumented launch needs a context");
    int rc = check_program(ctx, Prog::t, Prog::N, name);
    if (rc) return rc;
    rc = make_state(ctx, tools, &lc->st);
    if (rc) return rc;
    lc->stream = ctx->stream;
    NVBT_CUDA(cudaSetDevice(ctx->device));
  } else {
    lc->stream = ctx ? ctx->stream : static_cast<cudaStream_t>(stream);
  }
  return NVBT_OK;
}

static inline int done(nvbt_ctx ctx, int n_kernels) {
  NVBT_CUDA(cudaGetLastError());
  if (ctx) ctx->launches += n_kernels;
  return NVBT_OK;
}

}  // namespace nvbt
