// F4 — instruction emulation (paper §6.3; docs/EVENT_MODEL.md §3.6).
//
// NVBit's Device API lets a tool modify ISA-visible state; §6.3 uses it to emulate a hypothetical
// warp-wide 32-point FFT instruction WFFT32: the tool replaces the proxy instruction with a functionally
// equivalent device function wfft32emu() (Listing 9) and is combined with the instruction-count
// tool, to compare the instructions per warp of a kernel using WFFT32 (Listing 10) with the same
// FFT written in CUDA. Here the proxy site is compiled in: with NVBT_TOOL_EMU the site calls
// wfft32emu(); without it the proxy executes natively as a register move (X = x).
//
// Both programs compute the transform the same way (radix-2 decimation in frequency over warp shuffles,
// one complex element per lane, per-lane twiddles computed once per warp), so the emulated and the
// software kernel produce bit-identical fp32 results. The kernels are persistent: grid `ctas`, warp w
// handles transforms w, w + W, ... (W = 8 ctas). Inputs stream through a per-warp ring in shared memory
// (cp.async, 16 rows ahead) so each SM keeps enough bytes in flight to stream HBM without spending
// registers. Hooks are called in program order per loop instance (the virtual program
// of EM §3.6); only the data movement is pipelined.
#include "nvbt_internal.h"
#include "nvbt_workloads.h"
#include "programs.cuh"
#include "workload_launch.cuh"

namespace nvbt {

constexpr uint32_t TOOL_EMU = NVBT_TOOL_EMU;

// Per-lane constants of the transform (EM §3.6): stage signs, twiddles w_q(l), output lane brev5(l).
struct WfftLane {
  float sg[5];
  float wr[4], wi[4];
  unsigned rev;
};

// Hook sink for code that runs outside the virtual program (the emulation function's insides).
struct NoHooks {
  struct Act { unsigned A; };
  template <int PC>
  __device__ __forceinline__ void at(Act, bool = true, unsigned long long = 0) {}
};

// Twiddle setup of stage Q (pcs PC .. PC+7 of WFFT_SW): lanes with l & h set take
// w = exp(-2 pi i (l & (h-1)) 2^Q / 32) = (cospi(-k/16), sinpi(-k/16)), the others w = 1 and sign +1.
template <int Q, int PC, class H>
__device__ __forceinline__ void tw_stage(H& h, typename H::Act m, unsigned lane, WfftLane& c) {
  constexpr unsigned hh = 16u >> Q;
  const unsigned j = lane & (hh - 1u);          h.template at<PC>(m);
  const unsigned up = lane & hh;                h.template at<PC + 1>(m);
  const bool u = up != 0u;                      h.template at<PC + 2>(m);
  const float k = (float)(j << Q);              h.template at<PC + 3>(m);
  float s, co;
  sincospif(-k * 0.0625f, &s, &co);             h.template at<PC + 4>(m);
                                                h.template at<PC + 5>(m);
  c.wr[Q] = u ? co : 1.f;                       h.template at<PC + 6>(m);
  c.wi[Q] = u ? s : 0.f;                        h.template at<PC + 7>(m);
  c.sg[Q] = u ? -1.f : 1.f;
}

template <int PC, class H>
__device__ __forceinline__ void wfft_setup(H& h, typename H::Act m, unsigned lane, WfftLane& c) {
  tw_stage<0, PC>(h, m, lane, c);
  tw_stage<1, PC + 8>(h, m, lane, c);
  tw_stage<2, PC + 16>(h, m, lane, c);
  tw_stage<3, PC + 24>(h, m, lane, c);
  c.sg[4] = (lane & 1u) ? -1.f : 1.f;
  c.rev = __brev(lane);                         h.template at<PC + 32>(m);
  c.rev >>= 27;                                 h.template at<PC + 33>(m);
}

// DIF stage Q (span h = 16 >> Q; pcs PC .. PC+7, or PC .. PC+3 for Q = 4):
// d = xp + x (l & h == 0) or xp - x (l & h != 0), x = d * w_Q(l).
template <int Q, int PC, class H>
__device__ __forceinline__ void fft_stage(H& h, typename H::Act m, float& vr, float& vi, const WfftLane& c) {
  constexpr unsigned hh = 16u >> Q;
  const float pr = __shfl_xor_sync(FULL, vr, hh);   h.template at<PC>(m);
  const float pi = __shfl_xor_sync(FULL, vi, hh);   h.template at<PC + 1>(m);
  const float dr = __fmaf_rn(c.sg[Q], vr, pr);      h.template at<PC + 2>(m);
  const float di = __fmaf_rn(c.sg[Q], vi, pi);      h.template at<PC + 3>(m);
  if constexpr (Q < 4) {
    const float t = __fmul_rn(di, c.wi[Q]);          h.template at<PC + 4>(m);
    vr = __fmaf_rn(dr, c.wr[Q], -t);                 h.template at<PC + 5>(m);
    const float t2 = __fmul_rn(di, c.wr[Q]);         h.template at<PC + 6>(m);
    vi = __fmaf_rn(dr, c.wi[Q], t2);                 h.template at<PC + 7>(m);
  } else {
    vr = dr;
    vi = di;
  }
}

// The five stages; afterwards lane l holds X[brev5(l)].
template <int PC, class H>
__device__ __forceinline__ void fft_stages(H& h, typename H::Act m, float& vr, float& vi, const WfftLane& c) {
  fft_stage<0, PC>(h, m, vr, vi, c);
  fft_stage<1, PC + 8>(h, m, vr, vi, c);
  fft_stage<2, PC + 16>(h, m, vr, vi, c);
  fft_stage<3, PC + 24>(h, m, vr, vi, c);
  fft_stage<4, PC + 32>(h, m, vr, vi, c);
}

// Listing 9's wfft32emu(): functionally WFFT32 — lane k receives X[k] (natural order).
__device__ __forceinline__ float2 wfft32emu(float2 v, const WfftLane& c) {
  NoHooks nh;
  fft_stages<0>(nh, NoHooks::Act{0u}, v.x, v.y, c);
  v.x = __shfl_sync(FULL, v.x, c.rev);
  v.y = __shfl_sync(FULL, v.y, c.rev);
  return v;
}

// Per-warp copy ring: the input row of loop instance k lands in slot k % kRing of the warp's ring,
// kRing - 1 instances ahead of its use, through cp.async (16 B per lane, lanes 0-15 copy one 256 B row;
// one commit group per instance, so `cp.async.wait_group kRing - 1` is exactly "row k has landed").
// Bytes in flight per SM cost no registers: 8 warps x 16 slots x 256 B = 32 KB per CTA. Measured
// alternatives: a per-warp ring of 256 B cp.async.bulk copies with one mbarrier per slot (same bytes in
// flight, ~30 more instructions per transform for the barrier phase and the uniform-operand loop around
// the bulk copy: EMU|COUNT 1.94 ms), and a CTA-wide ring of 2 KB bulk stages with one producer warp (it
// couples the warps' progress: 2.18 ms).
constexpr int kRing = 16;
struct WfftRing {
  float2 slot[8][kRing][32];
};

__device__ __forceinline__ void ring_copy(unsigned lane, unsigned dst_row, const float2* src_row, bool on) {
  if (on && lane < 16u)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst_row + 16u * lane), "l"(src_row + 2u * lane)
                 : "memory");
  asm volatile("cp.async.commit_group;" ::: "memory");
}

template <uint32_t T, int V>
__global__ void __launch_bounds__(256) k_wfft(const float2* __restrict__ x, float2* __restrict__ X, int n_fft,
                                              int ctas, DevState st) {
  constexpr uint32_t TH = T & ~TOOL_EMU;
  constexpr bool kEmu = (T & TOOL_EMU) != 0;
  using Prog = std::conditional_t<V == 0, ProgWfftEmu, ProgWfftSw>;
  constexpr int LO = V == 0 ? 5 : 39;                 // loop body: first pc
  constexpr int S = V == 0 ? 8 : 77;                  // IMAD.WIDE before the store
  constexpr int EXIT_PC = V == 0 ? 13 : 82;
  __shared__ __align__(16) unsigned sb[Hooks<TH, Prog>::kSmemWords];
  __shared__ __align__(128) WfftRing ring;
  Hooks<TH, Prog> h(st, sb);
  const unsigned lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
  const auto m0 = h.active(true);
  const int tid = threadIdx.x;                        h.template at<0>(m0);
  const int cta = st.cta_lo + blockIdx.x;            h.template at<1>(m0);   // logical CTA (partition)
  const int f0 = cta * 8 + (tid >> 5);                h.template at<2>(m0);
  const bool p0 = f0 >= n_fft;                        h.template at<3>(m0);
                                                      h.template at<4>(m0, p0);  // @P0 EXIT (warp-uniform)
  const bool live = !p0;
  const auto m1 = h.active(live);
  if (live) {
    WfftLane c;
    if constexpr (V == 1) {
      wfft_setup<5>(h, m1, lane, c);
    } else if constexpr (kEmu) {
      NoHooks nh;
      wfft_setup<0>(nh, NoHooks::Act{0u}, lane, c);
    }
    const int W = ctas * 8;
    const int kw = (n_fft - f0 + W - 1) / W;          // loop instances of this warp (>= 1)
    const unsigned slot0 = (unsigned)__cvta_generic_to_shared(&ring.slot[wib][0][0]);
#pragma unroll
    for (int d = 0; d < kRing; ++d)
      ring_copy(lane, slot0 + 256u * d, x + (size_t)(f0 + d * W) * 32, d < kw);
    auto instance = [&](int k) {                      // warp-uniform: one loop instance per transform
      const int ff = f0 + k * W;
      const unsigned sl = (unsigned)k & (kRing - 1u);
      const float2* px = x + (size_t)ff * 32 + lane;        h.template at<LO>(m1);
      asm volatile("cp.async.wait_group %0;" ::"n"(kRing - 1) : "memory");   // row k has landed
      __syncwarp();
      float2 v;
      asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(slot0 + 256u * sl + 8u * lane) : "memory");
                                                             h.template at<LO + 1>(m1, true, (unsigned long long)px);
      unsigned col = lane;
      if constexpr (V == 0) {
        if constexpr (kEmu) v = wfft32emu(v, c);             // the tool replaces WFFT32 ...
                                                             // ... else the proxy is a register move
        h.template at<7>(m1);
      } else {
        fft_stages<41>(h, m1, v.x, v.y, c);
        col = c.rev;
      }
      float2* pX = X + (size_t)ff * 32 + col;                h.template at<S>(m1);
      __stcs(pX, v);                                         h.template at<S + 1>(m1, true, (unsigned long long)pX);
      // every lane's slot read has been consumed (the store used it): refill the slot with row k + kRing
      __syncwarp();
      ring_copy(lane, slot0 + 256u * sl, x + (size_t)(ff + kRing * W) * 32, k + kRing < kw);
                                                             h.template at<S + 2>(m1);
                                                             h.template at<S + 3>(m1);
                                                             h.template at<S + 4>(m1, k + 1 < kw);  // @P1 BRA
    };
    constexpr int kChunk = (int)decltype(h)::kSpillEvery;
    if (kw <= kChunk) {                               // the u32 counters cannot wrap: the plain loop
#pragma unroll 1
      for (int k = 0; k < kw; ++k) instance(k);
    } else {                                          // chunks of kChunk instances, counters spilled between
#pragma unroll 1
      for (int k0 = 0; k0 < kw; k0 += kChunk) {
        const int k1 = kw - k0 > kChunk ? k0 + kChunk : kw;
#pragma unroll 1
        for (int k = k0; k < k1; ++k) instance(k);
        if (k1 < kw) h.spill();
      }
    }
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  h.template at<EXIT_PC>(m1);
  h.finish();
}

template <class F>
static int dispatch_wfft(uint32_t tools, int variant, F&& f) {
  if (variant == NVBT_WFFT_SOFTWARE) {
    if (tools & TOOL_EMU) return set_error(NVBT_EINVAL, "NVBT_TOOL_EMU needs the proxy variant");
    return dispatch(tools, [&](auto tag) { f(tag, std::integral_constant<int, 1>{}); });
  }
  if (tools & TOOL_EMU)
    return dispatch(tools & ~TOOL_EMU, [&](auto tag) {
      f(std::integral_constant<uint32_t, decltype(tag)::value | TOOL_EMU>{}, std::integral_constant<int, 0>{});
    });
  return dispatch(tools, [&](auto tag) { f(tag, std::integral_constant<int, 0>{}); });
}

}  // namespace nvbt

using namespace nvbt;

extern "C" int nvbt_wfft32_max_ctas(uint32_t tools, int32_t variant, int32_t device, int32_t* ctas) {
  if (!ctas) return set_error(NVBT_EINVAL, "ctas is null");
  if (variant != NVBT_WFFT_PROXY && variant != NVBT_WFFT_SOFTWARE) return set_error(NVBT_EINVAL, "bad variant %d", variant);
  int sms = 0, per_sm = 0;
  NVBT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  cudaError_t err = cudaSuccess;
  const int rc = dispatch_wfft(tools, variant, [&](auto tag, auto var) {
    err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_wfft<decltype(tag)::value, decltype(var)::value>, 256, 0);
  });
  if (rc) return rc;
  NVBT_CUDA(err);
  *ctas = sms * per_sm;
  return NVBT_OK;
}

extern "C" int nvbt_wfft32(nvbt_ctx ctx, void* stream, uint32_t tools, int32_t variant, const void* x, void* X,
                           int32_t n_fft, int32_t ctas) {
  // (transform indices f + 5W stay below 2^31 in the kernel's int arithmetic)
  if (!x || !X || n_fft < 0 || ctas < 1 || (int64_t)n_fft + 40 * (int64_t)ctas >= (1ll << 31))
    return set_error(NVBT_EINVAL, "bad WFFT32 arguments");
  if (variant != NVBT_WFFT_PROXY && variant != NVBT_WFFT_SOFTWARE) return set_error(NVBT_EINVAL, "bad variant %d", variant);
  if (((uintptr_t)x | (uintptr_t)X) & 15u) return set_error(NVBT_EINVAL, "x and X must be 16-byte aligned");
  const char* xa = static_cast<const char*>(x);
  const char* Xa = static_cast<const char*>(X);
  if (xa < Xa + (size_t)n_fft * 256 && Xa < xa + (size_t)n_fft * 256 && n_fft > 0)
    return set_error(NVBT_EINVAL, "x and X overlap");
  const uint32_t instr = tools & ~TOOL_EMU;
  LaunchCtx lc;
  int rc = variant == NVBT_WFFT_PROXY ? prepare<ProgWfftEmu>(ctx, stream, instr, "WFFT_EMU", &lc)
                                      : prepare<ProgWfftSw>(ctx, stream, instr, "WFFT_SW", &lc);
  if (rc) return rc;
  if (ctx && instr == 0) lc.stream = ctx->stream;
  rc = partition(ctx, 1, (unsigned long long)ctas, &lc);
  if (rc) return rc;
  if (n_fft == 0 || lc.n_ctas == 0) return NVBT_OK;   // nothing launched (EM §3.6)
  rc = dispatch_wfft(tools, variant, [&](auto tag, auto var) {
    k_wfft<decltype(tag)::value, decltype(var)::value><<<lc.grid, 256, 0, lc.stream>>>(
        static_cast<const float2*>(x), static_cast<float2*>(X), n_fft, ctas, lc.st);
  });
  return rc ? rc : done(ctx, 1);
}
