/* nvbt synthetic workloads with compiled-in injection points (EM = docs/EVENT_MODEL.md §3).
 *
 * NVBit injects calls into SASS at run time (P:L123, P:L147-167 (§4, §5.1)); SASS decode and
 * trampolines are out of scope here, so each workload kernel is written once with a hook at every
 * injection point of its program table and compiled in several variants: `tools` (enum nvbt_tools)
 * picks the variant per launch, NVBT_TOOL_NONE being the same source with every hook compiled out
 * (the slowdown baseline). Conventions as in nvbt.h; all pointers are caller-owned device memory and
 * every launch is enqueued on the context's stream (asynchronous). Each instrumented launch takes the
 * next launch id ℓ of the context (EM §5).
 */
#ifndef NVBT_WORKLOADS_H
#define NVBT_WORKLOADS_H

#include "nvbt.h"

#ifdef __cplusplus
extern "C" {
#endif

enum nvbt_workload { NVBT_W_VECTORADD = 1, NVBT_W_SGEMM = 2, NVBT_W_BFS = 3, NVBT_W_STENCIL = 4,
                     NVBT_W_REPLAY = 5, NVBT_W_WFFT_EMU = 6, NVBT_W_WFFT_SW = 7 };

/* Copies a workload's program table (EM §3.1-3.5) into out[cap]; *n_pcs, *n_opcodes, *n_bbs receive
 * its sizes (any may be null). EINVAL if cap is too small (with *n_pcs still set). Host-only. */
int nvbt_program(int workload, nvbt_instr_desc* out, uint32_t cap, uint32_t* n_pcs,
                 uint32_t* n_opcodes, uint32_t* n_bbs);

/* Global warp count of one launch (for sizing PER_WARP contexts). Host-only.
 * args: VECTORADD {N}; SGEMM {M, N}; BFS {n}; STENCIL {n}; WFFT_EMU / WFFT_SW {n_fft, ctas}. */
int nvbt_workload_warps(int workload, const int64_t* args, uint32_t n_args, uint64_t* n_warps);

/* C1: c[i] = a[i] + b[i], i < N; CTA 256, grid ceil(N/256) (EM §3.1). ctx may be NULL when tools == 0
 * (then stream is used); otherwise the context's program must be the vectorAdd program. */
int nvbt_vectoradd(nvbt_ctx ctx, void* stream, uint32_t tools, const float* a, const float* b, float* c,
                   int32_t N);
/* C2: naive row-fastest SGEMM C[M,N] = A[M,K] B[K,N], fp32 row-major, K >= 1 (EM §3.2); ceil(N/8) <= 65535. */
int nvbt_sgemm(nvbt_ctx ctx, void* stream, uint32_t tools, const float* A, const float* B, float* C,
               int32_t M, int32_t N, int32_t K);
/* C3: one BFS level = kernel 1 (expand) then kernel 2 (update, writes cost = level + 1) (EM §3.3).
 * mask/visited/updating: u8[n]; cost: i32[n]; over: one i32 (kernel 2 stores 1 into it). The caller
 * zeroes *over and updating before the call (the host loop of EM §3.3). An instrumented expand over a
 * vertex of degree >= 2^24 would overflow the privatised u32 bins: it is flagged on the device and the
 * context's next read call returns NVBT_EINVAL (until nvbt_reset). SGEMM (any K) and WFFT32 (any n_fft)
 * spill their loop counters to the 64-bit bins every 2^20 instances instead. */
int nvbt_bfs_level(nvbt_ctx ctx, void* stream, uint32_t tools, const int32_t* rowptr, const int32_t* col,
                   int32_t n, uint8_t* mask, uint8_t* visited, uint8_t* updating, int32_t* cost,
                   int32_t* over, int32_t level);
/* C3 kernels 1 (expand) and 2 (update) as separate launches, for a multi-GPU BFS that exchanges
 * `updating` between them and `visited` / `over` after kernel 2. Same arguments and launch
 * ids as the two halves of nvbt_bfs_level. */
int nvbt_bfs_expand(nvbt_ctx ctx, void* stream, uint32_t tools, const int32_t* rowptr, const int32_t* col,
                    int32_t n, uint8_t* mask, const uint8_t* visited, uint8_t* updating);
int nvbt_bfs_update(nvbt_ctx ctx, void* stream, uint32_t tools, int32_t n, uint8_t* mask, uint8_t* visited,
                    uint8_t* updating, int32_t* cost, int32_t* over, int32_t level);
/* C4: one Jacobi iteration out = stencil(in) on an n x n fp32 grid (EM §3.4); ceil(n/8) <= 65535. */
int nvbt_stencil(nvbt_ctx ctx, void* stream, uint32_t tools, const float* in, float* out, int32_t n);

/* Multi-GPU partition ("partitioned ... by kernel and warp range"): every later workload
 * launch through ctx (C1-C4 and F4; not replay, whose event ranges are explicit) runs only rank's share
 * of its CTA grid. A grid of gy rows of gx CTAs (2D workloads: SGEMM and stencil, gx = ceil(M/32) resp.
 * ceil(n/32); 1D workloads: gx = 1, gy = CTAs) gives rank r of `world` the whole CTA rows
 * [floor(gy r / world), floor(gy (r + 1) / world)). Warp ids, addresses and events are those of the
 * unpartitioned launch (the kernels use the logical CTA id), so the world ranks' accumulators sum to the
 * single-GPU result (EM §4) and each rank writes only its share of the outputs. A rank with an empty
 * share still takes the launch id. Default: rank 0 of 1. EINVAL if world == 0 or rank >= world. */
int nvbt_set_partition(nvbt_ctx ctx, uint32_t rank, uint32_t world);

/* F4, instruction emulation (§6.3; EM §3.6): n_fft warp-wide 32-point FFTs.
 * x, X: caller-owned device arrays of n_fft x 32 complex64 (interleaved fp32 re, im; 256 B per transform,
 * 16 B aligned), x and X must not overlap. CTA 256 threads, grid `ctas` (>= 1; part of the event model:
 * warp w computes transforms w, w + 8 ctas, ...). variant NVBT_WFFT_PROXY runs program WFFT_EMU (the
 * kernel using the hypothetical WFFT32 instruction, Listing 10 analogue): with NVBT_TOOL_EMU in `tools`
 * the instruction is replaced by its emulation function (Listing 9's wfft32emu: lane k receives
 * X[k] = sum_n x[n] exp(-2 pi i n k / 32)); without it the proxy executes natively as a 64-bit register
 * move, so X = x. variant NVBT_WFFT_SOFTWARE runs program WFFT_SW (the same transform written in CUDA,
 * radix-2 DIF over warp shuffles; NVBT_TOOL_EMU is EINVAL there). Both compute bit-identical transforms
 * in fp32. The other tool bits instrument the launch as for every workload (ctx must hold the matching
 * program); tools in {0, NVBT_TOOL_EMU} need no context (stream is used). */
enum nvbt_wfft_variant { NVBT_WFFT_PROXY = 0, NVBT_WFFT_SOFTWARE = 1 };
int nvbt_wfft32(nvbt_ctx ctx, void* stream, uint32_t tools, int32_t variant, const void* x, void* X,
                int32_t n_fft, int32_t ctas);
/* *ctas = SMs of `device` x resident CTAs per SM of the kernel that (tools, variant) selects: the grid
 * that keeps every warp of a persistent launch resident (one wave). EINVAL as nvbt_wfft32 for tools. */
int nvbt_wfft32_max_ctas(uint32_t tools, int32_t variant, int32_t device, int32_t* ctas);

#ifdef __cplusplus
}
#endif
#endif
