// Host-side internals of libnvbt.so (context, workspace layout, error reporting).
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <mutex>
#include <string>
#include <vector>

#include "nvbt.h"
#include "nvbt_hooks.cuh"

namespace nvbt {

int set_error(int code, const char* fmt, ...);
#define NVBT_CUDA(call)                                                                      \
  do {                                                                                      \
    cudaError_t e_ = (call);                                                                \
    if (e_ != cudaSuccess)                                                                  \
      return ::nvbt::set_error(NVBT_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), \
                               __FILE__, __LINE__);                                         \
  } while (0)

// Workspace layout (bytes from d_workspace). The accumulator region comes first and is one packed
// int64 array: K stripes of {site[4P] | bbsite[4P] | mem[3P] | hist[66]}, then pw[2W]. A CTA flushes its
// shared bins into stripe (linear CTA id % K), so kernels with many small CTAs do not serialise on the
// same global addresses; the fold kernel sums the stripes (integer sums, order-free).
struct Layout {
  size_t site, bbsite, mem, hist, pw, accum_words;   // word offsets into the accumulator region
  size_t stripe_words, stripes;                     // site..hist repeat `stripes` times (CTA-striped bins)
  size_t ctl;                                       // byte offsets from here on
  size_t prog, leader, kind, out;
  size_t out_words;
  size_t total;
  // out (fold result) word offsets
  size_t o_counts, o_ht, o_hw, o_bb, o_mem, o_memtot, o_hist;
};
Layout make_layout(uint32_t n_pcs, uint32_t n_ops, uint32_t n_bbs, uint32_t n_warps, uint32_t flags);

// CTL_RHEAD: device-ring (F2) region heads, kMaxRingStripes stripes + 1 overflow region
constexpr unsigned kMaxRingStripes = 255;
enum Ctl { CTL_HEAD = 0, CTL_TAIL_CACHE = 1, CTL_DROPPED = 2, CTL_REPLAY_ERR = 3, CTL_OVERFLOW = 4, CTL_RHEAD = 8,
           CTL_WORDS = 8 + kMaxRingStripes + 1 };

}  // namespace nvbt

struct nvbt_chan_s;

struct nvbt_ctx_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  uint32_t n_pcs = 0, n_ops = 0, n_bbs = 0, n_warps = 0, flags = 0;
  std::vector<nvbt_instr_desc> prog;
  nvbt::Layout lay{};
  unsigned char* ws = nullptr;
  unsigned long long* accum = nullptr;
  unsigned long long* ctl = nullptr;
  unsigned long long* out = nullptr;
  nvbt_instr_desc* d_prog = nullptr;
  uint32_t* d_leader = nullptr;
  uint8_t* d_kind = nullptr;
  uint32_t next_launch = 0;
  uint32_t part_rank = 0, part_world = 1;   // nvbt_set_partition
  std::atomic<uint64_t> launches{0};
  nvbt_chan_s* chan = nullptr;
  std::mutex mu;

  unsigned long long* site() const { return accum + lay.site; }
  unsigned long long* bbsite() const { return accum + lay.bbsite; }
  unsigned long long* mem() const { return accum + lay.mem; }
  unsigned long long* hist() const { return accum + lay.hist; }
  unsigned long long* pw() const { return (flags & NVBT_PER_WARP) ? accum + lay.pw : nullptr; }
};

namespace nvbt {
// Builds the DevState for one instrumented launch with `tools`; validates tools against the context.
int make_state(nvbt_ctx ctx, uint32_t tools, DevState* st);
// Checks that the context's program is `prog[n]`.
int check_program(nvbt_ctx ctx, const nvbt_instr_desc* prog, int n, const char* name);
void channel_state(nvbt_chan_s* ch, DevState* st);
bool channel_open(nvbt_chan_s* ch);
int fold(nvbt_ctx ctx);  // runs the fold kernel and copies the result to host-visible staging
// Per-device facts and one-time function attributes (both are per device: a process may drive several
// GPUs). device_sms: SM count of `dev`, cached. func_smem: cudaFuncSetAttribute(MaxDynamicSharedMemorySize)
// once per (function, device), errors reported as NVBT_ECUDA.
int device_sms(int dev);
int func_smem(const void* fn, int dev, size_t bytes);
// Loads every workload kernel variant on `dev` once (cudaFuncGetAttributes), so no first launch lazily loads
// a module while a trace producer waits on the host consumer: under CUDA_MODULE_LOADING=LAZY, loading a
// kernel may synchronise the context, i.e. wait for a producer that waits for the drain (nvbt_channel_open).
int preload_workload_kernels(int dev);
}  // namespace nvbt
