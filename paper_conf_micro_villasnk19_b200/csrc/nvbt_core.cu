// libnvbt.so core: context lifecycle, workspace layout, the fold kernel and the read calls (nvbt.h).
#include <algorithm>
#include <cstring>
#include <new>

#include "nvbt_internal.h"

namespace nvbt {

static thread_local std::string g_err;

int set_error(int code, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

Layout make_layout(uint32_t P, uint32_t O, uint32_t B, uint32_t W, uint32_t flags) {
  Layout L{};
  L.site = 0;
  L.bbsite = L.site + 4ull * P;
  L.mem = L.bbsite + 4ull * P;
  L.hist = L.mem + 3ull * P;
  L.stripe_words = L.hist + 66;
  L.stripes = P <= 64 ? 32 : 1;   // small programs (the workloads) run many small CTAs
  L.pw = L.stripe_words * L.stripes;
  L.accum_words = L.pw + ((flags & NVBT_PER_WARP) ? 2ull * W : 0);
  size_t off = align_up(L.accum_words * 8, 256);
  L.ctl = off;
  off = align_up(off + CTL_WORDS * 8, 256);
  L.prog = off;
  off = align_up(off + sizeof(nvbt_instr_desc) * P, 256);
  L.leader = off;
  off = align_up(off + 4ull * B, 256);
  L.kind = off;
  off = align_up(off + P, 256);
  L.out = off;
  L.o_counts = 0;
  L.o_ht = 4;
  L.o_hw = L.o_ht + O;
  L.o_bb = L.o_hw + O;
  L.o_mem = L.o_bb + 4ull * B;
  L.o_memtot = L.o_mem + 3ull * P;
  L.o_hist = L.o_memtot + 3;
  L.out_words = L.o_hist + 66;
  off = align_up(off + L.out_words * 8, 256);
  L.total = off;
  return L;
}

// ---------------------------------------------------------------------------------------------------
// Fold kernel: per-pc bins (per-instruction mode + BB mode derived per EM §2 item 3) -> reported
// counts, opcode histogram, BB statistics and divergence totals. Integer sums only.
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// One warp per pc; lane s sums stripes s, s+32, ... of the CTA-striped bins.
__global__ void fold_kernel(const nvbt_instr_desc* __restrict__ prog, const uint32_t* __restrict__ leader,
                            uint32_t P, uint32_t O, uint32_t B, const unsigned long long* __restrict__ accum,
                            unsigned long long* out, Layout L) {
  const size_t SW = L.stripe_words;
  const unsigned lane = threadIdx.x & 31u;
  const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t pc = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; pc < P; pc += warps) {
    const nvbt_instr_desc d = prog[pc];
    const uint32_t l = leader[d.bb];
    unsigned long long tI = 0, tE = 0, wI = 0, wE = 0, n = 0, sS = 0, sL = 0;
    for (size_t s = lane; s < L.stripes; s += 32) {
      const unsigned long long* site = accum + s * SW + L.site;
      const unsigned long long* bbsite = accum + s * SW + L.bbsite;
      const unsigned long long* mem = accum + s * SW + L.mem;
      tI += site[4 * pc]; tE += site[4 * pc + 1]; wI += site[4 * pc + 2]; wE += site[4 * pc + 3];
      if (d.is_leader || d.guarded) {
        tI += bbsite[4 * pc]; tE += bbsite[4 * pc + 1]; wI += bbsite[4 * pc + 2]; wE += bbsite[4 * pc + 3];
      } else {  // same active mask as the block's leader (BB rule), unguarded: E = A
        tI += bbsite[4 * l]; tE += bbsite[4 * l]; wI += bbsite[4 * l + 2]; wE += bbsite[4 * l + 2];
      }
      n += mem[3 * pc]; sS += mem[3 * pc + 1]; sL += mem[3 * pc + 2];
    }
    tI = warp_sum_u64(tI); tE = warp_sum_u64(tE); wI = warp_sum_u64(wI); wE = warp_sum_u64(wE);
    n = warp_sum_u64(n); sS = warp_sum_u64(sS); sL = warp_sum_u64(sL);
    if (lane == 0) {
      if (tI | wI) {
        atomicAdd(out + L.o_counts + 0, tI);
        atomicAdd(out + L.o_counts + 1, tE);
        atomicAdd(out + L.o_counts + 2, wI);
        atomicAdd(out + L.o_counts + 3, wE);
        atomicAdd(out + L.o_ht + d.opcode, tE);
        atomicAdd(out + L.o_hw + d.opcode, wE);
        unsigned long long* bb = out + L.o_bb + 4ull * d.bb;
        if (d.is_leader) { atomicAdd(bb + 0, wI); atomicAdd(bb + 1, tI); }
        atomicAdd(bb + 2, wE);
        atomicAdd(bb + 3, tE);
      }
      out[L.o_mem + 3 * pc] = n;
      out[L.o_mem + 3 * pc + 1] = sS;
      out[L.o_mem + 3 * pc + 2] = sL;
      if (n) {
        atomicAdd(out + L.o_memtot, n);
        atomicAdd(out + L.o_memtot + 1, sS);
        atomicAdd(out + L.o_memtot + 2, sL);
      }
    }
  }
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t < 66) {
    unsigned long long h = 0;
    for (size_t s = 0; s < L.stripes; ++s) h += accum[s * SW + L.hist + t];
    out[L.o_hist + t] = h;
  }
}

int device_sms(int dev) {
  static std::mutex m;
  static std::vector<int> sms;
  std::lock_guard<std::mutex> g(m);
  if (dev < 0) return 148;
  if ((size_t)dev >= sms.size()) sms.resize((size_t)dev + 1, 0);
  if (sms[dev] == 0) cudaDeviceGetAttribute(&sms[dev], cudaDevAttrMultiProcessorCount, dev);
  return sms[dev] > 0 ? sms[dev] : 148;
}

int func_smem(const void* fn, int dev, size_t bytes) {
  static std::mutex m;
  static std::vector<std::pair<const void*, int>> done;   // (function, device) pairs already set
  std::lock_guard<std::mutex> g(m);
  for (auto& d : done)
    if (d.first == fn && d.second == dev) return NVBT_OK;
  const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e != cudaSuccess)
    return set_error(NVBT_ECUDA, "cudaFuncSetAttribute(%zu B dynamic shared) on device %d: %s", bytes, dev,
                     cudaGetErrorString(e));
  done.emplace_back(fn, dev);
  return NVBT_OK;
}

int fold(nvbt_ctx c) {
  NVBT_CUDA(cudaSetDevice(c->device));
  NVBT_CUDA(cudaMemsetAsync(c->out, 0, c->lay.out_words * 8, c->stream));
  const int threads = 256;
  const int blocks = (int)std::min<uint32_t>((c->n_pcs + 7) / 8, 1184);   // 8 warps (pcs) per block
  fold_kernel<<<blocks, threads, 0, c->stream>>>(c->d_prog, c->d_leader, c->n_pcs, c->n_ops, c->n_bbs, c->accum,
                                                  c->out, c->lay);
  NVBT_CUDA(cudaGetLastError());
  c->launches++;
  return NVBT_OK;
}

__global__ void axpy_kernel(unsigned long long* __restrict__ y, const unsigned long long* __restrict__ x, size_t n,
                            unsigned long long a) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    y[i] += a * x[i];
}

static int read_out(nvbt_ctx c, size_t word, size_t n, void* dst) {
  std::lock_guard<std::mutex> g(c->mu);
  int rc = fold(c);
  if (rc) return rc;
  unsigned long long ovf = 0;
  NVBT_CUDA(cudaMemcpyAsync(dst, c->out + word, n * 8, cudaMemcpyDeviceToHost, c->stream));
  NVBT_CUDA(cudaMemcpyAsync(&ovf, c->ctl + CTL_OVERFLOW, 8, cudaMemcpyDeviceToHost, c->stream));
  NVBT_CUDA(cudaStreamSynchronize(c->stream));
  if (ovf)
    return set_error(NVBT_EINVAL, "%llu warp(s) ran a loop of >= 2^24 instances (a BFS vertex of degree >= 2^24): "
                     "their u32 CTA bins could wrap, results withheld until nvbt_reset", ovf);
  return NVBT_OK;
}

int make_state(nvbt_ctx c, uint32_t tools, DevState* st) {
  if ((tools & NVBT_TOOL_COUNT) && (tools & NVBT_TOOL_BBCOUNT))
    return set_error(NVBT_EINVAL, "tools: COUNT and BBCOUNT are exclusive");
  if (tools & ~uint32_t(15)) return set_error(NVBT_EINVAL, "tools: unknown bits 0x%x", tools);
  if ((tools & (NVBT_TOOL_COUNT | NVBT_TOOL_BBCOUNT)) && !(c->flags & (NVBT_COUNT | NVBT_OPHIST | NVBT_BB)))
    return set_error(NVBT_ESTATE, "counting tool needs NVBT_COUNT/OPHIST/BB at init");
  if ((tools & NVBT_TOOL_MEMDIV) && !(c->flags & NVBT_MEMDIV))
    return set_error(NVBT_ESTATE, "memdiv tool needs NVBT_MEMDIV at init");
  if (tools & NVBT_TOOL_TRACE) {
    if (!(c->flags & NVBT_TRACE)) return set_error(NVBT_ESTATE, "trace tool needs NVBT_TRACE at init");
    if (c->chan == nullptr || !channel_open(c->chan)) return set_error(NVBT_ESTATE, "trace tool needs an open channel");
  }
  std::memset(st, 0, sizeof *st);
  st->site = (tools & NVBT_TOOL_BBCOUNT) ? c->bbsite() : c->site();
  st->mem = c->mem();
  st->hist = c->hist();
  st->pw = c->pw();
  st->n_warps = c->n_warps;
  st->stripes = (unsigned)c->lay.stripes;
  st->stripe_words = c->lay.stripe_words;
  st->head = c->ctl + CTL_HEAD;
  st->tail_cache = c->ctl + CTL_TAIL_CACHE;
  st->dropped = c->ctl + CTL_DROPPED;
  st->ovf = c->ctl + CTL_OVERFLOW;
  if ((tools & NVBT_TOOL_TRACE) && c->chan) channel_state(c->chan, st);
  st->launch = c->next_launch++;
  return NVBT_OK;
}

int check_program(nvbt_ctx c, const nvbt_instr_desc* prog, int n, const char* name) {
  if ((int)c->n_pcs != n || std::memcmp(c->prog.data(), prog, sizeof(nvbt_instr_desc) * n) != 0)
    return set_error(NVBT_EINVAL, "context program is not the %s program", name);
  return NVBT_OK;
}

}  // namespace nvbt

using namespace nvbt;

extern "C" {

int nvbt_abi_version(void) { return NVBT_ABI_VERSION; }
const char* nvbt_last_error(void) { return g_err.c_str(); }

static int validate_sizes(const nvbt_config* cfg) {
  if (!cfg) return set_error(NVBT_EINVAL, "cfg is null");
  if (cfg->version != NVBT_ABI_VERSION)
    return set_error(NVBT_EVERSION, "ABI version %u, library has %d", cfg->version, NVBT_ABI_VERSION);
  if (cfg->n_pcs == 0 || cfg->n_pcs > 4096) return set_error(NVBT_EINVAL, "n_pcs %u not in 1..4096", cfg->n_pcs);
  if (cfg->n_opcodes == 0 || cfg->n_opcodes > 256) return set_error(NVBT_EINVAL, "n_opcodes %u not in 1..256", cfg->n_opcodes);
  if (cfg->n_bbs == 0 || cfg->n_bbs > cfg->n_pcs) return set_error(NVBT_EINVAL, "n_bbs %u not in 1..n_pcs", cfg->n_bbs);
  if ((cfg->flags & NVBT_PER_WARP) && cfg->n_warps == 0) return set_error(NVBT_EINVAL, "PER_WARP needs n_warps > 0");
  if (cfg->flags & ~uint32_t(63)) return set_error(NVBT_EINVAL, "unknown flag bits 0x%x", cfg->flags);
  return NVBT_OK;
}

int nvbt_workspace_size(const nvbt_config* cfg, size_t* bytes) {
  int rc = validate_sizes(cfg);
  if (rc) return rc;
  if (!bytes) return set_error(NVBT_EINVAL, "bytes is null");
  *bytes = make_layout(cfg->n_pcs, cfg->n_opcodes, cfg->n_bbs, cfg->n_warps, cfg->flags).total;
  return NVBT_OK;
}

int nvbt_init(const nvbt_config* cfg, nvbt_ctx* out) {
  int rc = validate_sizes(cfg);
  if (rc) return rc;
  if (!out || !cfg->prog || !cfg->d_workspace) return set_error(NVBT_EINVAL, "null prog, workspace or out");
  if (reinterpret_cast<uintptr_t>(cfg->d_workspace) % 256) return set_error(NVBT_EINVAL, "workspace not 256-byte aligned");
  Layout L = make_layout(cfg->n_pcs, cfg->n_opcodes, cfg->n_bbs, cfg->n_warps, cfg->flags);
  if (cfg->workspace_bytes < L.total)
    return set_error(NVBT_ENOMEM, "workspace %zu bytes < %zu needed", cfg->workspace_bytes, L.total);
  // program table checks (EM §3): ids in range, bb ids non-decreasing, leaders exactly at bb starts
  std::vector<uint32_t> leader(cfg->n_bbs, UINT32_MAX);
  std::vector<uint8_t> kind(cfg->n_pcs);
  for (uint32_t pc = 0; pc < cfg->n_pcs; ++pc) {
    const nvbt_instr_desc& d = cfg->prog[pc];
    if (d.opcode >= cfg->n_opcodes) return set_error(NVBT_EINVAL, "pc %u: opcode %u >= n_opcodes", pc, d.opcode);
    if (d.bb >= cfg->n_bbs) return set_error(NVBT_EINVAL, "pc %u: bb %u >= n_bbs", pc, d.bb);
    if (d.kind > NVBT_K_OTHERMEM) return set_error(NVBT_EINVAL, "pc %u: kind %u", pc, d.kind);
    const bool starts = pc == 0 || cfg->prog[pc - 1].bb != d.bb;
    if (starts != (d.is_leader != 0)) return set_error(NVBT_EINVAL, "pc %u: is_leader does not mark a block start", pc);
    if (pc > 0 && d.bb < cfg->prog[pc - 1].bb) return set_error(NVBT_EINVAL, "pc %u: bb ids must be non-decreasing", pc);
    if (is_mem_kind(d.kind) && (d.width == 0 || (d.width & (d.width - 1)) || d.width > 128))
      return set_error(NVBT_EINVAL, "pc %u: memory width %u", pc, d.width);
    if (d.is_leader) leader[d.bb] = pc;
    kind[pc] = d.kind;
  }
  for (uint32_t b = 0; b < cfg->n_bbs; ++b)
    if (leader[b] == UINT32_MAX) return set_error(NVBT_EINVAL, "bb %u has no instructions", b);

  nvbt_ctx c = new (std::nothrow) nvbt_ctx_s();
  if (!c) return set_error(NVBT_ENOMEM, "host allocation failed");
  c->device = cfg->device;
  c->stream = static_cast<cudaStream_t>(cfg->stream);
  c->n_pcs = cfg->n_pcs; c->n_ops = cfg->n_opcodes; c->n_bbs = cfg->n_bbs; c->n_warps = cfg->n_warps;
  c->flags = cfg->flags;
  c->prog.assign(cfg->prog, cfg->prog + cfg->n_pcs);
  c->lay = L;
  c->ws = static_cast<unsigned char*>(cfg->d_workspace);
  c->accum = reinterpret_cast<unsigned long long*>(c->ws);
  c->ctl = reinterpret_cast<unsigned long long*>(c->ws + L.ctl);
  c->d_prog = reinterpret_cast<nvbt_instr_desc*>(c->ws + L.prog);
  c->d_leader = reinterpret_cast<uint32_t*>(c->ws + L.leader);
  c->d_kind = reinterpret_cast<uint8_t*>(c->ws + L.kind);
  c->out = reinterpret_cast<unsigned long long*>(c->ws + L.out);
  auto fail = [&](int code) { delete c; return code; };
  if (cudaSetDevice(c->device) != cudaSuccess) return fail(set_error(NVBT_ECUDA, "cudaSetDevice(%d) failed", c->device));
  cudaPointerAttributes pa{};
  if (cudaPointerGetAttributes(&pa, cfg->d_workspace) != cudaSuccess || pa.type != cudaMemoryTypeDevice)
    return fail(set_error(NVBT_EINVAL, "workspace is not device memory"));
  if (cudaMemsetAsync(c->ws, 0, L.total, c->stream) != cudaSuccess ||
      cudaMemcpyAsync(c->d_prog, cfg->prog, sizeof(nvbt_instr_desc) * cfg->n_pcs, cudaMemcpyHostToDevice, c->stream) != cudaSuccess ||
      cudaMemcpyAsync(c->d_leader, leader.data(), 4ull * cfg->n_bbs, cudaMemcpyHostToDevice, c->stream) != cudaSuccess ||
      cudaMemcpyAsync(c->d_kind, kind.data(), cfg->n_pcs, cudaMemcpyHostToDevice, c->stream) != cudaSuccess ||
      cudaStreamSynchronize(c->stream) != cudaSuccess)
    return fail(set_error(NVBT_ECUDA, "workspace upload failed: %s", cudaGetErrorString(cudaGetLastError())));
  *out = c;
  return NVBT_OK;
}

int nvbt_reset(nvbt_ctx c) {
  if (!c) return set_error(NVBT_EINVAL, "ctx is null");
  std::lock_guard<std::mutex> g(c->mu);
  NVBT_CUDA(cudaSetDevice(c->device));
  NVBT_CUDA(cudaMemsetAsync(c->accum, 0, c->lay.accum_words * 8, c->stream));
  NVBT_CUDA(cudaMemsetAsync(c->ctl + CTL_REPLAY_ERR, 0, 16, c->stream));   // replay errors, overflow
  c->next_launch = 0;
  return NVBT_OK;
}

int nvbt_fini(nvbt_ctx c) {
  if (!c) return set_error(NVBT_EINVAL, "ctx is null");
  if (c->chan) nvbt_channel_close(c->chan);
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->stream);
  delete c;
  return NVBT_OK;
}

int nvbt_accum_view(nvbt_ctx c, void** d_ptr, size_t* n) {
  if (!c || !d_ptr || !n) return set_error(NVBT_EINVAL, "null argument");
  *d_ptr = c->accum;
  *n = c->lay.accum_words;
  return NVBT_OK;
}

int nvbt_accum_axpy(nvbt_ctx c, const void* d_src, size_t n, int64_t factor) {
  if (!c || (!d_src && n)) return set_error(NVBT_EINVAL, "null argument");
  if (n != c->lay.accum_words) return set_error(NVBT_EINVAL, "n_int64 %zu != accumulator words %zu", n, c->lay.accum_words);
  if (factor < 0) return set_error(NVBT_EINVAL, "factor must be >= 0");
  if (n == 0 || factor == 0) return NVBT_OK;
  NVBT_CUDA(cudaSetDevice(c->device));
  const int blocks = (int)std::min<size_t>((n + 255) / 256, 1024);
  axpy_kernel<<<blocks, 256, 0, c->stream>>>(c->accum, static_cast<const unsigned long long*>(d_src), n,
                                             (unsigned long long)factor);
  NVBT_CUDA(cudaGetLastError());
  c->launches++;
  return NVBT_OK;
}

int nvbt_count(nvbt_ctx c, nvbt_counts* out, uint64_t* pwt, uint64_t* pww) {
  if (!c || !out) return set_error(NVBT_EINVAL, "null argument");
  if (!(c->flags & (NVBT_COUNT | NVBT_OPHIST | NVBT_BB))) return set_error(NVBT_ESTATE, "NVBT_COUNT not enabled");
  if ((pwt || pww) && !(c->flags & NVBT_PER_WARP)) return set_error(NVBT_ESTATE, "NVBT_PER_WARP not enabled");
  uint64_t v[4];
  int rc = read_out(c, c->lay.o_counts, 4, v);
  if (rc) return rc;
  out->thread_issued = v[0]; out->thread_exec = v[1]; out->warp_issued = v[2]; out->warp_exec = v[3];
  if (pwt) NVBT_CUDA(cudaMemcpy(pwt, c->accum + c->lay.pw, 8ull * c->n_warps, cudaMemcpyDeviceToHost));
  if (pww) NVBT_CUDA(cudaMemcpy(pww, c->accum + c->lay.pw + c->n_warps, 8ull * c->n_warps, cudaMemcpyDeviceToHost));
  return NVBT_OK;
}

int nvbt_opcode_hist(nvbt_ctx c, uint64_t* t, uint64_t* w, uint32_t n) {
  if (!c || !t || !w) return set_error(NVBT_EINVAL, "null argument");
  if (n != c->n_ops) return set_error(NVBT_EINVAL, "n_opcodes %u != context's %u", n, c->n_ops);
  if (!(c->flags & (NVBT_OPHIST | NVBT_COUNT))) return set_error(NVBT_ESTATE, "NVBT_OPHIST not enabled");
  std::vector<uint64_t> v(2ull * n);
  int rc = read_out(c, c->lay.o_ht, 2ull * n, v.data());
  if (rc) return rc;
  std::memcpy(t, v.data(), 8ull * n);
  std::memcpy(w, v.data() + n, 8ull * n);
  return NVBT_OK;
}

int nvbt_bb_count(nvbt_ctx c, nvbt_bb_stats* out, uint32_t n) {
  if (!c || !out) return set_error(NVBT_EINVAL, "null argument");
  if (n != c->n_bbs) return set_error(NVBT_EINVAL, "n_bbs %u != context's %u", n, c->n_bbs);
  if (!(c->flags & (NVBT_BB | NVBT_COUNT))) return set_error(NVBT_ESTATE, "NVBT_BB not enabled");
  static_assert(sizeof(nvbt_bb_stats) == 32, "layout");
  return read_out(c, c->lay.o_bb, 4ull * n, out);
}

int nvbt_mem_divergence(nvbt_ctx c, nvbt_memdiv* per_pc, uint32_t n, nvbt_memdiv_total* tot) {
  if (!c || !tot) return set_error(NVBT_EINVAL, "null argument");
  if (!(c->flags & NVBT_MEMDIV)) return set_error(NVBT_ESTATE, "NVBT_MEMDIV not enabled");
  if (per_pc && n != c->n_pcs) return set_error(NVBT_EINVAL, "n_pcs %u != context's %u", n, c->n_pcs);
  std::vector<uint64_t> v(3ull * c->n_pcs + 3 + 66);
  int rc = read_out(c, c->lay.o_mem, v.size(), v.data());
  if (rc) return rc;
  if (per_pc) std::memcpy(per_pc, v.data(), 24ull * c->n_pcs);
  const uint64_t* t = v.data() + 3ull * c->n_pcs;
  tot->sum.accesses = t[0]; tot->sum.sectors = t[1]; tot->sum.lines = t[2];
  std::memcpy(tot->hist_sectors, t + 3, 33 * 8);
  std::memcpy(tot->hist_lines, t + 36, 33 * 8);
  return NVBT_OK;
}

int nvbt_replay_errors(nvbt_ctx c, uint64_t* bad) {
  if (!c || !bad) return set_error(NVBT_EINVAL, "null argument");
  NVBT_CUDA(cudaMemcpyAsync(bad, c->ctl + CTL_REPLAY_ERR, 8, cudaMemcpyDeviceToHost, c->stream));
  NVBT_CUDA(cudaStreamSynchronize(c->stream));
  return NVBT_OK;
}

int nvbt_device_state(nvbt_ctx c, uint32_t tools, void* out_pod, size_t pod_bytes) {
  if (!c || !out_pod) return set_error(NVBT_EINVAL, "null argument");
  if (pod_bytes != sizeof(nvbt_dev_state))
    return set_error(NVBT_EINVAL, "pod_bytes %zu != sizeof(nvbt_dev_state) %zu", pod_bytes, sizeof(nvbt_dev_state));
  if (tools & (NVBT_TOOL_TRACE | NVBT_TOOL_EMU))
    return set_error(NVBT_EINVAL, "external kernels get COUNT / BBCOUNT / MEMDIV hooks only");
  std::lock_guard<std::mutex> g(c->mu);
  DevState st;
  int rc = make_state(c, tools, &st);
  if (rc) return rc;
  nvbt_dev_state d{};
  d.version = NVBT_DEV_STATE_VERSION;
  d.tools = tools;
  d.site = st.site;
  d.mem = st.mem;
  d.hist = st.hist;
  d.per_warp = st.pw;
  d.stripe_words = st.stripe_words;
  d.stripes = st.stripes;
  d.n_pcs = c->n_pcs;
  d.n_warps = st.pw ? c->n_warps : 0;
  d.launch = st.launch;
  std::memcpy(out_pod, &d, sizeof d);
  return NVBT_OK;
}

int nvbt_launch_count(nvbt_ctx c, uint64_t* n) {
  if (!c || !n) return set_error(NVBT_EINVAL, "null argument");
  *n = c->launches.load();
  return NVBT_OK;
}

}  // extern "C"
