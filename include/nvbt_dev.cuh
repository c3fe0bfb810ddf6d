/* nvbt public device API (include/nvbt_dev.cuh): the compiled-in analogue of NVBit's injected device
 * functions, for kernels OUTSIDE libnvbt.so.
 *
 * NVBit injects a call before a SASS instruction and passes it the guard predicate, register values and
 * immediates (nvbit_insert_call / nvbit_add_call_arg, P:L123 (§4); Listing 8, P:L243-246 (§6.1)); the
 * injected function then runs for every active thread (P:L307 (§7)). SASS decode and injection are out of
 * scope here (north_star), so a kernel calls these hooks itself at its injection points, with the pc of
 * the instruction in the program table its context was created with (nvbt_config.prog, the stand-in for
 * NVBit's Instr objects). Results land in that context's accumulators and are read with
 * nvbt_count / nvbt_opcode_hist / nvbt_bb_count / nvbt_mem_divergence (include/nvbt.h), exactly as for
 * the library's own workloads (docs/EVENT_MODEL.md §2).
 *
 * Usage (all 32 lanes of every warp call every hook — lanes that exited or are on another path pass
 * in_flow = false; the "converged-hook discipline", R-15):
 *
 *   #include "nvbt_dev.cuh"                          // nvcc -I include, sm_100a
 *   __global__ void k(nvbt_dev_state st, ...) {
 *     extern __shared__ unsigned char smem[];        // NVBT_DEV_SMEM_BYTES(n_pcs, warps per CTA)
 *     nvbt_hooks h;
 *     nvbt_cta_begin(h, st, smem);                   // every thread of the CTA (contains __syncthreads)
 *     ...
 *     nvbt_on_instr(h, 4, live, i >= n);             // counting hook at pc 4 (guarded)
 *     nvbt_on_mem(h, 7, live, true, (uint64_t)&x[i]);// divergence hook at a global LD/ST
 *     ...
 *     nvbt_cta_flush(h);                             // every thread of the CTA, once, at the end
 *   }
 *   host: nvbt_device_state(ctx, NVBT_TOOL_COUNT | NVBT_TOOL_MEMDIV, &st, sizeof st); k<<<g, b, smem>>>(st, ...);
 *
 * Hooks (the tools of nvbt_device_state decide what the counting hooks record):
 *   nvbt_on_instr(h, pc, in_flow, pred)       counting at one instruction. NVBT_TOOL_COUNT: call it at every
 *                                             pc. NVBT_TOOL_BBCOUNT: call it only at GUARDED non-leader pcs
 *                                             (the per-pc counts of the others follow from the block's
 *                                             entries, P:L89 (§3), P:L115-117 (§4)).
 *   nvbt_on_bb(h, pc, in_flow, len, pred)     NVBT_TOOL_BBCOUNT: at the first instruction (pc) of a basic
 *                                             block of len instructions; pred = that instruction's guard.
 *   nvbt_on_mem(h, pc, in_flow, pred, addr)   NVBT_TOOL_MEMDIV: distinct 32 B sectors and 128 B lines of a
 *                                             warp-level global LD/ST (Listing 8).
 *                                             Counting at the same pc is a separate call (NVBit also allows
 *                                             several injected calls per instruction).
 *   nvbt_cta_flush(h)                         CTA epilogue: shared bins -> the context's global bins, one
 *                                             64-bit atomic per non-zero bin (P:L89's per-block counters).
 * Event formation (EM §1): A = ballot(in_flow), P = ballot(in_flow && pred) (P is A's subset), E = A & P
 * ("a false predicate value means that the instrumented instruction is not actually executing").
 * All CTA bins are 64-bit, so no count can wrap. Shared memory: NVBT_DEV_SMEM_BYTES(P, W) = 8 (7 P + 66) +
 * 768 W bytes (about 7 KB for P = 64 pcs and 8 warps); programs beyond ~3,900 pcs do not fit one CTA. Warp ids for the per-warp arrays are EM §1's
 * linear_cta * warps_per_cta + tid_linear / 32; the CTA must hold a whole number of warps.
 */
#pragma once
#include <cstdint>
#include "nvbt.h"

namespace nvbt {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ unsigned lane_id() { unsigned l; asm("mov.u32 %0, %%laneid;" : "=r"(l)); return l; }
__device__ __forceinline__ unsigned smid() { unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s)); return s; }
__device__ __forceinline__ unsigned lanemask_lt() { unsigned m; asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m)); return m; }
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t;
}

__host__ __device__ constexpr bool is_mem_kind(int k) { return k == NVBT_K_GLD || k == NVBT_K_GST || k == NVBT_K_GATOM; }

// Number of distinct keys among the lanes of E with __match_any_sync (kept for comparison; MATCH's
// cost grows with the number of distinct keys, so the hot path uses sectors_lines() below).
__device__ __forceinline__ unsigned distinct_match(unsigned long long key, unsigned E, unsigned lanebit, unsigned lmlt) {
  const unsigned grp = __match_any_sync(FULL, key);
  return __popc(__ballot_sync(FULL, (E & lanebit) != 0u && (grp & E & lmlt) == 0u));
}

#ifndef NVBT_AP_FASTPATH
#define NVBT_AP_FASTPATH 1
#endif
constexpr int SCRATCH_WORDS = 192;  // per-warp scratch of sectors_lines(): 64 x u64 keys + 64 x u32 masks
// Initial contents of scratch word i (keys empty = ~0, masks 0).
__host__ __device__ constexpr unsigned scratch_init_word(int i) { return i < 128 ? 0xffffffffu : 0u; }

// Slow paths of sectors_lines() (addresses not non-decreasing in lane order), cheapest first; `scr` is
// the warp's shared scratch (SCRATCH_WORDS words in their initial state, restored before returning):
//  * every sector in the first lane's 32-sector (1 KB) word: OR-reduce one bit per sector;
//    S = popc, L = popc of the OR-ed 4-bit groups;
//  * every sector within a 1024-sector (32 KB) window: a 32-word shared bitmap, same counts;
//  * all lines distinct (hashed 4096-bucket occupancy == |E|): S = L = |E|;
//  * otherwise a per-warp open-addressing hash set of LINE keys: each lane of E inserts its line with a
//    64-bit CAS (linear probing, 64 slots >= 2 x 32 keys), then ORs its sector's bit into the slot's
//    4-bit mask; L = lanes that inserted, S = sum of mask popcounts.
__device__ __forceinline__ unsigned lds_u32_(unsigned a) {
  unsigned v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ uint2 sectors_lines_unsorted(unsigned long long addr, unsigned E, unsigned lane,
                                                        unsigned lanebit, unsigned scr) {
  const bool act = (E & lanebit) != 0u;
  const unsigned long long sk = addr >> 5;
  const unsigned long long sk0 = __shfl_sync(FULL, sk, __ffs(E) - 1);
  if (__all_sync(FULL, !act || (sk >> 5) == (sk0 >> 5))) {
    const unsigned word = __reduce_or_sync(FULL, act ? 1u << (unsigned)(sk & 31) : 0u);
    const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
    return make_uint2(__popc(word), __popc(g & 0x11111111u));
  }
  // 32 KB window around the first lane's sector: clear one bit per sector in the 32 "key" words (kept
  // at ~0 between uses, so the same area doubles as the hash table's empty keys)
  const long long wv = (long long)(sk - (sk0 & ~31ull)) + 512;
  if (__all_sync(FULL, !act || (wv >= 0 && wv < 1024))) {
    if (act) asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(scr + 4u * (unsigned)(wv >> 5)), "r"(~(1u << (unsigned)(wv & 31))) : "memory");
    __syncwarp();
    const unsigned word = ~lds_u32_(scr + 4u * lane);
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(scr + 4u * lane), "r"(0xffffffffu) : "memory");
    __syncwarp();
    const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
    return make_uint2(__reduce_add_sync(FULL, __popc(word)), __reduce_add_sync(FULL, __popc(g & 0x11111111u)));
  }
  const unsigned long long line = sk >> 2;
  const unsigned hh = ((unsigned)line ^ (unsigned)(line >> 32)) * 0x9E3779B1u;
  // all lines distinct? (wide random addresses): 4096-bucket hashed bitmap in the 128 key words. No
  // bucket shared => all lines and hence all sectors distinct => S = L = |E|; else exact hash set below
  if (act) asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(scr + 4u * (hh >> 25)), "r"(~(1u << ((hh >> 20) & 31u))) : "memory");
  __syncwarp();
  {
    unsigned w0, w1, w2, w3;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(w0), "=r"(w1), "=r"(w2), "=r"(w3) : "r"(scr + 16u * lane) : "memory");
    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(scr + 16u * lane), "r"(0xffffffffu) : "memory");
    const unsigned used = __reduce_add_sync(FULL, __popc(~w0) + __popc(~w1) + __popc(~w2) + __popc(~w3));
    __syncwarp();
    if (used == (unsigned)__popc(E)) return make_uint2(used, used);
  }
  unsigned slot = hh >> 26;
  bool pending = act, inserted = false;
  while (__any_sync(FULL, pending)) {
    if (pending) {
      unsigned long long old;
      asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(scr + 8u * slot), "l"(~0ull), "l"(line)
                   : "memory");
      if (old == ~0ull || old == line) {
        pending = false;
        inserted = old == ~0ull;
      } else {
        slot = (slot + 1u) & 63u;
      }
    }
  }
  if (act) asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(scr + 512u + 4u * slot), "r"(1u << (unsigned)(sk & 3)) : "memory");
  const unsigned L = __popc(__ballot_sync(FULL, inserted));
  __syncwarp();
  unsigned m0, m1;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(m0), "=r"(m1) : "r"(scr + 512u + 8u * lane) : "memory");
  asm volatile("st.shared.v2.u32 [%0], {%1, %1};" ::"r"(scr + 512u + 8u * lane), "r"(0u) : "memory");
  asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(scr + 16u * lane), "r"(0xffffffffu) : "memory");
  const unsigned S = __reduce_add_sync(FULL, __popc(m0) + __popc(m1));
  __syncwarp();
  return make_uint2(S, L);
}
// The same S/L for a caller that has already classified the access (the staged replay's lane scan knows
// the minimum and maximum address of E): cls 0 = every address in one 1 KB word, cls 1 = every sector in
// the 1024-sector window starting at sector `wbase` (32-aligned; all upper address words equal), cls 2 =
// anything else (hashed all-distinct test, then the hash set). Same scratch contract as above.
__device__ __forceinline__ uint2 sectors_lines_cls(unsigned long long addr, unsigned E, unsigned lanebit,
                                                   unsigned lane, unsigned scr, unsigned cls, unsigned wbase) {
  const bool act = (E & lanebit) != 0u;
  const unsigned sk_lo = (unsigned)(addr >> 5);
  if (cls == 0u) {
    const unsigned word = __reduce_or_sync(FULL, act ? 1u << (sk_lo & 31u) : 0u);
    const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
    return make_uint2(__popc(word), __popc(g & 0x11111111u));
  }
  if (cls == 1u) {
    const unsigned wv = ((unsigned)addr >> 5) - wbase;   // upper words equal: the low word orders the window
    if (act) asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(scr + 4u * (wv >> 5)), "r"(~(1u << (wv & 31u))) : "memory");
    __syncwarp();
    const unsigned word = ~lds_u32_(scr + 4u * lane);
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(scr + 4u * lane), "r"(0xffffffffu) : "memory");
    __syncwarp();
    const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
    return make_uint2(__reduce_add_sync(FULL, __popc(word)), __reduce_add_sync(FULL, __popc(g & 0x11111111u)));
  }
  const unsigned long long line = addr >> 7;
  const unsigned hh = ((unsigned)line ^ (unsigned)(line >> 32)) * 0x9E3779B1u;
  if (act) asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(scr + 4u * (hh >> 25)), "r"(~(1u << ((hh >> 20) & 31u))) : "memory");
  __syncwarp();
  {
    unsigned w0, w1, w2, w3;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(w0), "=r"(w1), "=r"(w2), "=r"(w3) : "r"(scr + 16u * lane) : "memory");
    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(scr + 16u * lane), "r"(0xffffffffu) : "memory");
    const unsigned used = __reduce_add_sync(FULL, __popc(~w0) + __popc(~w1) + __popc(~w2) + __popc(~w3));
    __syncwarp();
    if (used == (unsigned)__popc(E)) return make_uint2(used, used);
  }
  unsigned slot = hh >> 26;
  bool pending = act, inserted = false;
  while (__any_sync(FULL, pending)) {
    if (pending) {
      unsigned long long old;
      asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(scr + 8u * slot), "l"(~0ull), "l"(line)
                   : "memory");
      if (old == ~0ull || old == line) {
        pending = false;
        inserted = old == ~0ull;
      } else {
        slot = (slot + 1u) & 63u;
      }
    }
  }
  if (act) asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(scr + 512u + 4u * slot), "r"(1u << (sk_lo & 3u)) : "memory");
  const unsigned L = __popc(__ballot_sync(FULL, inserted));
  __syncwarp();
  unsigned m0, m1;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(m0), "=r"(m1) : "r"(scr + 512u + 8u * lane) : "memory");
  asm volatile("st.shared.v2.u32 [%0], {%1, %1};" ::"r"(scr + 512u + 8u * lane), "r"(0u) : "memory");
  asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(scr + 16u * lane), "r"(0xffffffffu) : "memory");
  const unsigned S = __reduce_add_sync(FULL, __popc(m0) + __popc(m1));
  __syncwarp();
  return make_uint2(S, L);
}

// The three classes of sectors_lines_cls() as separate functions (callers that loop per class):
// sl_word: all lanes of E in one 1 KB word (only the low address word is needed);
__device__ __forceinline__ uint2 sl_word(unsigned a_lo, bool act) {
  const unsigned word = __reduce_or_sync(FULL, act ? 1u << ((a_lo >> 5) & 31u) : 0u);
  const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
  return make_uint2(__popc(word), __popc(g & 0x11111111u));
}
// sl_window: all sectors of E in the 1024-sector window from sector wbase (32-aligned, upper words equal);
__device__ __forceinline__ uint2 sl_window(unsigned a_lo, bool act, unsigned lane, unsigned scr, unsigned wbase) {
  const unsigned wv = (a_lo >> 5) - wbase;
  if (act) asm volatile("red.shared.and.b32 [%0], %1;" ::"r"(scr + 4u * (wv >> 5)), "r"(~(1u << (wv & 31u))) : "memory");
  __syncwarp();
  const unsigned word = ~lds_u32_(scr + 4u * lane);
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(scr + 4u * lane), "r"(0xffffffffu) : "memory");
  __syncwarp();
  const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
  return make_uint2(__reduce_add_sync(FULL, __popc(word)), __reduce_add_sync(FULL, __popc(g & 0x11111111u)));
}
// sl_wide: anything else (class 2 of sectors_lines_cls).
__device__ __forceinline__ uint2 sl_wide(unsigned long long addr, unsigned E, unsigned lanebit, unsigned lane,
                                         unsigned scr) {
  return sectors_lines_cls(addr, E, lanebit, lane, scr, 2u, 0u);
}

static __device__ __noinline__ uint2 sectors_lines_unsorted_call(unsigned long long addr, unsigned E, unsigned lane,
                                                                 unsigned lanebit, unsigned scr) {
  return sectors_lines_unsorted(addr, E, lane, lanebit, scr);
}

// a5 kernel of Listing 8 (readings R-3, R-5, R-6): S = number of distinct 32 B
// sectors and L = number of distinct 128 B lines touched by the lanes of E (E != 0). Exact integers.
// Fast paths (coalesced, strided, broadcast, stencil neighbours ...): when the addresses of the lanes of
// E are non-decreasing in lane order, so are their sectors and lines, and each distinct value starts
// where a lane's sector (line) differs from the previous lane of E — compared as (a ^ prev) >> 5 (7).
// kApFirst: for a full warp, first try an arithmetic progression a_l = min + l d detected with warp
// reductions (no shuffles: the instrumented application kernels are L1-bound, and shuffles share the
// L1/MIO datapath with their loads), whose S and L have a closed form in (min, max, d); otherwise the
// previous lane's address comes from 2 shuffles.
// Other orders take the slow paths above (inlined when kInlineSlow, else an out-of-line call to keep the
// hooks' registers and code small).
template <bool kInlineSlow = false, bool kApFirst = true>
__device__ __forceinline__ void sectors_lines(unsigned long long addr, unsigned E, unsigned lane, unsigned lanebit,
                                              unsigned lmlt, unsigned scr, unsigned& S, unsigned& L) {
  const unsigned a_lo = (unsigned)addr, a_hi = (unsigned)(addr >> 32);
#if NVBT_AP_FASTPATH
  if (kApFirst && E == FULL) {
    // all 32 lanes, addresses an increasing arithmetic progression in lane order inside one 4 GB
    // region (coalesced, strided, broadcast): warp reductions instead of shuffles — a_l = min + l d
    const unsigned hmn = __reduce_min_sync(FULL, a_hi), hmx = __reduce_max_sync(FULL, a_hi);
    const unsigned mn = __reduce_min_sync(FULL, a_lo), mx = __reduce_max_sync(FULL, a_lo);
    const unsigned dd = (mx - mn) / 31u;
    if (hmn == hmx && __all_sync(FULL, a_lo == mn + lane * dd)) {
      // closed form, warp-uniform arithmetic only: a step d < 32 (< 128) can skip no sector (line), so
      // the distinct sectors (lines) are every one from mn's to mx's; a step >= 32 (>= 128) puts every
      // lane in its own sector (line)
      S = dd >= 32u ? 32u : (mx >> 5) - (mn >> 5) + 1u;
      L = dd >= 128u ? 32u : (mx >> 7) - (mn >> 7) + 1u;
      return;
    }
  }
#endif
  const unsigned below = E & lmlt;
  unsigned src;                                    // previous lane of E (0xffffffff -> lane 31: unused)
  asm("bfind.u32 %0, %1;" : "=r"(src) : "r"(below));
  unsigned p_lo = __shfl_sync(FULL, a_lo, src), p_hi = __shfl_sync(FULL, a_hi, src);
  // lanes outside E and the first lane of E compare with themselves: no boundary, no violation
  const bool take = (E & lanebit) != 0u && below != 0u;
  p_lo = take ? p_lo : a_lo;
  p_hi = take ? p_hi : a_hi;
  const long long d = (long long)(((unsigned long long)a_hi << 32 | a_lo) - ((unsigned long long)p_hi << 32 | p_lo));
  if (__all_sync(FULL, d >= 0)) {
    const unsigned x_lo = a_lo ^ p_lo, x_hi = a_hi ^ p_hi;
    S = 1u + __popc(__ballot_sync(FULL, ((x_lo & ~31u) | x_hi) != 0u));
    L = 1u + __popc(__ballot_sync(FULL, ((x_lo & ~127u) | x_hi) != 0u));
    return;
  }
  const uint2 r = kInlineSlow ? sectors_lines_unsorted(addr, E, lane, lanebit, scr)
                              : sectors_lines_unsorted_call(addr, E, lane, lanebit, scr);
  S = r.x;
  L = r.y;
}

__device__ __forceinline__ unsigned umin(unsigned a, unsigned b) { return a < b ? a : b; }
// h += (v == ref) as a predicated add.
__device__ __forceinline__ void inc_if_eq(unsigned& h, unsigned v, unsigned ref) {
  asm("{\n\t.reg .pred p;\n\tsetp.eq.u32 p, %1, %2;\n\t@p add.u32 %0, %0, 1;\n\t}" : "+r"(h) : "r"(v), "r"(ref));
}

}  // namespace nvbt

/* ---------------------------------------------------------------------------------------------------
 * Public hooks. */
#define NVBT_DEV_BIN_WORDS 7   /* per pc: t_issued, t_exec, w_issued, w_exec, n, sectors, lines (u64) */
/* dynamic shared memory a CTA needs for n_pcs program counters and `warps` warps */
#define NVBT_DEV_SMEM_BYTES(n_pcs, warps) (8ull * ((n_pcs) * NVBT_DEV_BIN_WORDS + 66) + 4ull * nvbt::SCRATCH_WORDS * (warps))

struct nvbt_hooks {
  nvbt_dev_state st;
  unsigned long long* bins;   /* shared: [n_pcs][7] then hist [66] */
  unsigned scr;               /* shared address of this warp's divergence scratch */
  unsigned lane, lanebit, lmlt, gwarp;
  unsigned long long pwT, pwW;
};

__device__ __forceinline__ void nvbt_check_converged_() {
#ifdef NVBT_CHECK_CONVERGED
  if (__activemask() != nvbt::FULL) __trap();
#endif
}

/* Every thread of the CTA, before any hook. smem: NVBT_DEV_SMEM_BYTES(st.n_pcs, warps per CTA) bytes of
 * shared memory, 16-byte aligned. */
__device__ __forceinline__ void nvbt_cta_begin(nvbt_hooks& h, const nvbt_dev_state& st, void* smem) {
  h.st = st;
  h.bins = static_cast<unsigned long long*>(smem);
  const unsigned tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const unsigned nthreads = blockDim.x * blockDim.y * blockDim.z;
  const unsigned warps = nthreads >> 5;
  h.lane = nvbt::lane_id();
  h.lanebit = 1u << h.lane;
  h.lmlt = nvbt::lanemask_lt();
  const unsigned cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  h.gwarp = cta * warps + (tid >> 5);
  h.pwT = h.pwW = 0;
  const unsigned nb = st.n_pcs * NVBT_DEV_BIN_WORDS + 66;
  for (unsigned i = tid; i < nb; i += nthreads) h.bins[i] = 0ull;
  unsigned* scr = reinterpret_cast<unsigned*>(h.bins + nb);
  for (unsigned i = tid; i < nvbt::SCRATCH_WORDS * warps; i += nthreads) scr[i] = nvbt::scratch_init_word((int)(i % nvbt::SCRATCH_WORDS));
  h.scr = (unsigned)__cvta_generic_to_shared(scr + nvbt::SCRATCH_WORDS * (tid >> 5));
  __syncthreads();
}

/* counting at one instruction: t_issued += popc(A), t_exec += popc(E), w_issued += 1, w_exec += (E != 0) */
__device__ __forceinline__ void nvbt_count_event_(nvbt_hooks& h, uint32_t pc, unsigned A, unsigned E) {
  if (h.lane == 0) {
    unsigned long long* b = h.bins + NVBT_DEV_BIN_WORDS * pc;
    atomicAdd(b + 0, (unsigned long long)__popc(A));
    if (E) {
      atomicAdd(b + 1, (unsigned long long)__popc(E));
      atomicAdd(b + 3, 1ull);
    }
    atomicAdd(b + 2, 1ull);
  }
}

__device__ __forceinline__ void nvbt_on_instr(nvbt_hooks& h, uint32_t pc, bool in_flow, bool pred = true) {
  nvbt_check_converged_();
  const unsigned A = __ballot_sync(nvbt::FULL, in_flow);
  if (A == 0u) return;                                       /* EM §1: no event */
  const unsigned E = __ballot_sync(nvbt::FULL, in_flow && pred);
  nvbt_count_event_(h, pc, A, E);
  const unsigned pa = __popc(A), pe = __popc(E);
  if (h.st.tools & NVBT_TOOL_BBCOUNT) {                      /* guarded pc inside a block: the block's */
    h.pwT -= pa - pe;                                        /* entry already counted it as executed   */
    h.pwW -= (E == 0u) ? 1u : 0u;
  } else {
    h.pwT += pe;
    h.pwW += (E != 0u) ? 1u : 0u;
  }
}

__device__ __forceinline__ void nvbt_on_bb(nvbt_hooks& h, uint32_t pc, bool in_flow, uint32_t len, bool pred = true) {
  nvbt_check_converged_();
  const unsigned A = __ballot_sync(nvbt::FULL, in_flow);
  if (A == 0u) return;
  const unsigned E = __ballot_sync(nvbt::FULL, in_flow && pred);
  nvbt_count_event_(h, pc, A, E);
  const unsigned pa = __popc(A), pe = __popc(E);
  h.pwT += (unsigned long long)len * pa - (pa - pe);         /* every entered thread runs the block, */
  h.pwW += len - ((E == 0u) ? 1u : 0u);                      /* the leader's guard aside    */
}

__device__ __forceinline__ void nvbt_on_mem(nvbt_hooks& h, uint32_t pc, bool in_flow, bool pred, uint64_t addr) {
  nvbt_check_converged_();
  const unsigned E = __ballot_sync(nvbt::FULL, in_flow && pred);
  if (E == 0u) return;                                       /* R-10: no divergence for E = 0 */
  unsigned S, L;
  nvbt::sectors_lines<true, true>(addr, E, h.lane, h.lanebit, h.lmlt, h.scr, S, L);
  if (h.lane == 0) {
    unsigned long long* b = h.bins + NVBT_DEV_BIN_WORDS * pc;
    atomicAdd(b + 4, 1ull);
    atomicAdd(b + 5, (unsigned long long)S);
    atomicAdd(b + 6, (unsigned long long)L);
    unsigned long long* hist = h.bins + NVBT_DEV_BIN_WORDS * h.st.n_pcs;
    atomicAdd(hist + S, 1ull);
    atomicAdd(hist + 33 + L, 1ull);
  }
}

/* Every thread of the CTA, once, after its last hook. */
__device__ __forceinline__ void nvbt_cta_flush(nvbt_hooks& h) {
  const nvbt_dev_state& st = h.st;
  if (st.per_warp != nullptr && h.lane == 0 && h.gwarp < st.n_warps) {
    atomicAdd(st.per_warp + h.gwarp, h.pwT);
    atomicAdd(st.per_warp + st.n_warps + h.gwarp, h.pwW);
  }
  __syncthreads();
  const unsigned tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const unsigned nthreads = blockDim.x * blockDim.y * blockDim.z;
  const unsigned cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  const unsigned long long so = (unsigned long long)(cta & (st.stripes - 1u)) * st.stripe_words;
  for (unsigned i = tid; i < st.n_pcs * NVBT_DEV_BIN_WORDS; i += nthreads) {
    const unsigned long long v = h.bins[i];
    if (v == 0ull) continue;
    const unsigned pc = i / NVBT_DEV_BIN_WORDS, k = i % NVBT_DEV_BIN_WORDS;
    if (k < 4) atomicAdd(st.site + so + 4ull * pc + k, v);
    else atomicAdd(st.mem + so + 3ull * pc + (k - 4), v);
  }
  const unsigned long long* hist = h.bins + NVBT_DEV_BIN_WORDS * st.n_pcs;
  for (unsigned i = tid; i < 66; i += nthreads)
    if (hist[i]) atomicAdd(st.hist + so + i, hist[i]);
}
