// Trace-replay mode (a7) and its counter-based event generator (EM §3.5), plus nvbt_program().
//
// Replay applies EM §2 items 1-4 to an HBM-resident stream of 16 B event headers and 256 B address
// slots. It is HBM-bound: the algorithmic bytes are 16 per header plus 256 per executed memory event
// (the only slots that must be read). Two paths, same results:
//   * nvbt_replay (k_replay4): one pass, one CTA of 32 warps per SM; each warp strides over 32-event tiles
//     (lane l owns header tile*32+l), counts into per-CTA shared per-pc bins (folded into the global u64
//     bins once per CTA, a8), and analyses the tile's executed memory events warp-cooperatively
//     (sectors_lines(), slots staged by cp.async);
//   * nvbt_replay_staged (k_rpA + k_rpB): a header pass that lists the executed memory events and a slot
//     pass that analyses them lane-parallel from double-buffered shared stages (section below).
#include <cstdlib>
#include <cstring>


#include "nvbt_internal.h"
#include "nvbt_workloads.h"
#include "programs.cuh"

namespace nvbt {

// ---------------------------------------------------------------- generator (EM §3.5)
constexpr unsigned long long kSeed = 0x4E5642544E564254ull;
constexpr unsigned long long kFStep = 0xD1B54A32D192ED03ull;

__host__ __device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ unsigned long long Kf(unsigned long long seed, unsigned long long f) {
  return mix64(seed ^ (f * kFStep));
}

struct GenConsts {
  unsigned long long k[9];  // K(0..8); K(64 + lane) is computed per lane
  unsigned long long seed;
};

__global__ void __launch_bounds__(256) k_gen(GenConsts G, unsigned long long first, unsigned long long n,
                                             const uint8_t* __restrict__ kind, const nvbt_instr_desc* __restrict__ prog,
                                             uint4* __restrict__ hdr, unsigned long long* __restrict__ addr) {
  const unsigned lane = lane_id();
  const unsigned long long klane = Kf(G.seed, 64 + lane);
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  for (unsigned long long tile = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; tile * 32 < n; tile += warps) {
    const unsigned long long li = tile * 32 + lane;
    const bool valid = li < n;
    const unsigned long long i = first + li;
    const unsigned pc = (unsigned)(mix64(G.k[0] ^ i) & 4095ull);
    const unsigned warp = (unsigned)(mix64(G.k[1] ^ i) & ((1ull << 20) - 1));
    unsigned A = (mix64(G.k[2] ^ i) % 4 != 0) ? 0xffffffffu : (unsigned)mix64(G.k[3] ^ i);
    if (A == 0) A = 1;
    const unsigned P = (mix64(G.k[4] ^ i) % 8 < 6) ? 0xffffffffu : (unsigned)mix64(G.k[5] ^ i);
    if (valid) hdr[li] = make_uint4(pc, warp, A, P);
    const bool mem = valid && is_mem_kind(kind[pc]);
    unsigned pat = 0;
    unsigned long long base = 0, s = 0;
    if (mem) {
      pat = (unsigned)(mix64(G.k[6] ^ i) % 6);
      base = (mix64(G.k[7] ^ i) & ((1ull << 40) - 1)) & ~127ull;
      s = mix64(G.k[8] ^ i);
    }
    unsigned mm = __ballot_sync(FULL, mem);
    while (mm) {
      const int src = __ffs(mm) - 1;
      mm &= mm - 1;
      const unsigned long long is = __shfl_sync(FULL, i, src);
      const unsigned ps = __shfl_sync(FULL, pc, src);
      const unsigned pt = __shfl_sync(FULL, pat, src);
      const unsigned long long b = __shfl_sync(FULL, base, src);
      const unsigned long long ss = __shfl_sync(FULL, s, src);
      const unsigned long long wd = prog[ps].width;
      // R(i, 64 + lane) only for the two random patterns (pt is warp-uniform: no divergence)
      const unsigned long long r = (pt == 3u || pt == 4u) ? mix64(klane ^ is) : 0ull;
      unsigned long long a;
      switch (pt) {
        case 0: a = b + lane * wd; break;
        case 1: a = b + lane * (wd << (ss % 10)); break;
        case 2: a = b; break;
        case 3: a = b + (r % (4096 / wd)) * wd; break;
        case 4: a = (r & ((1ull << 40) - 1)) & ~(wd - 1); break;
        default: a = b + (lane ^ (unsigned)(ss & 31)) * wd; break;
      }
      addr[(tile * 32 + src) * 32 + lane] = a;
    }
  }
}

// ---------------------------------------------------------------- replay
__device__ __forceinline__ void red_shared_add(unsigned saddr, unsigned v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}
__device__ __forceinline__ void red_shared_add_if(bool p, unsigned saddr, unsigned v) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.shared.add.u32 [%0], %1;\n\t}"
               ::"r"(saddr), "r"(v), "r"((unsigned)p) : "memory");
}
__device__ __forceinline__ uint4 ld_nc_v4(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// shared-memory helpers (32-bit shared addresses)
__device__ __forceinline__ void lds_v4(unsigned a, uint4& v) {
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
}
__device__ __forceinline__ unsigned lds_u32(unsigned a) {
  unsigned v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts_u32(unsigned a, unsigned v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_u64(unsigned a, unsigned long long v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}

// ---------------------------------------------------------------- single-pass replay (nvbt_replay)
// One CTA of 32 warps per SM. Per 32-event tile: predicated shared reductions for the counts (no
// branches), then the tile's executed memory events in batches of 8: cp.async (8 B per lane) stages the
// 8 address slots into the warp's shared rows, and a rolled loop runs sectors_lines() per event with
// every shared access through explicit 32-bit shared addresses and predicated reductions (compact code:
// the I-cache holds the whole loop).
constexpr int L4_NW = 32;  // warps per CTA (1 CTA per SM)
constexpr int L4_WARP_WORDS = SCRATCH_WORDS + 4 + 8 * 64 + 32;   // scratch + pad + 8 stage rows + row sources

__device__ __forceinline__ void sts_u8(unsigned a, unsigned v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned lds_u8(unsigned a) {
  unsigned v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}

template <bool PW>
__global__ void __launch_bounds__(32 * L4_NW, 1)
k_replay4(const uint4* __restrict__ hdr, const unsigned long long* __restrict__ addr, unsigned long long n,
          unsigned P, const uint8_t* __restrict__ kind, DevState st, unsigned long long* err) {
  extern __shared__ __align__(16) unsigned sm[];
  const unsigned P4 = (6 * P + 66 + 3) & ~3u;
  unsigned* sWarpAll = sm + P4;
  uint8_t* sK = reinterpret_cast<uint8_t*>(sm + P4 + L4_NW * L4_WARP_WORDS);
  for (unsigned i = threadIdx.x; i < P4; i += blockDim.x) sm[i] = 0;
  for (unsigned i = threadIdx.x; i < L4_NW * L4_WARP_WORDS; i += blockDim.x) {
    const unsigned o = i % L4_WARP_WORDS;
    sWarpAll[i] = o < SCRATCH_WORDS ? scratch_init_word(o) : 0u;
  }
  for (unsigned i = threadIdx.x; i < P; i += blockDim.x) sK[i] = is_mem_kind(kind[i]);
  __syncthreads();

  const unsigned lane = lane_id(), lmlt = lanemask_lt(), lanebit = 1u << lane;
  const unsigned s_base = (unsigned)__cvta_generic_to_shared(sm);
  const unsigned s_kind = (unsigned)__cvta_generic_to_shared(sK);
  const unsigned s_scr = (unsigned)__cvta_generic_to_shared(sWarpAll + (threadIdx.x >> 5) * L4_WARP_WORDS);
  const unsigned s_stage0 = s_scr + 4u * SCRATCH_WORDS + 16u;          // row r at + 256 r
  const unsigned s_rowsrc = s_stage0 + 8u * 256u;                       // [32] lane of the r-th event
  const unsigned s_sS = s_base + 16u * P, s_sL = s_base + 20u * P;
  unsigned hS = 0, hL = 0, bad = 0;
  const unsigned long long warps = (unsigned long long)gridDim.x * L4_NW;
  unsigned long long tile = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
  uint4 h = make_uint4(0, 0, 0, 0);
  if (tile * 32 + lane < n) h = ld_nc_v4(hdr + tile * 32 + lane);
  for (; tile * 32 < n; tile += warps) {
    const bool valid = tile * 32 + lane < n;
    const unsigned pc = h.x, A = h.z, E = h.z & h.w;
    const unsigned long long nt = tile + warps;
    uint4 hn = make_uint4(0, 0, 0, 0);
    if (nt * 32 + lane < n) hn = ld_nc_v4(hdr + nt * 32 + lane);
    const bool ok = valid && pc < P && A != 0u;
    bad += valid && pc >= P;
    const unsigned pcs = ok ? pc : 0u;
    const unsigned a4 = s_base + 4u * pcs;
    const unsigned pa = __popc(A), pe = __popc(E);
    red_shared_add_if(ok, a4, pa);
    red_shared_add_if(ok, a4 + 4u * P, 1u);
    red_shared_add_if(ok && pa != pe, a4 + 8u * P, pa - pe);
    red_shared_add_if(ok && E == 0u, a4 + 12u * P, 1u);
    if constexpr (PW) {
      const unsigned warp = h.y;
      if (ok && warp < st.n_warps) {
        atomicAdd(st.pw + warp, (unsigned long long)pe);
        if (E) atomicAdd(st.pw + st.n_warps + warp, 1ull);
      }
    }
    const unsigned mm = __ballot_sync(FULL, ok && E != 0u && lds_u8(s_kind + pcs) != 0u);
    const unsigned long long* tbase0 = addr + tile * 32 * 32;
    const unsigned total = __popc(mm);
    if (total) {
      // row r of the tile's memory events = the r-th set lane of mm (each owner writes its lane id)
      if ((mm >> lane) & 1u) sts_u32(s_rowsrc + 4u * __popc(mm & lmlt), lane);
      __syncwarp();
    }
    for (unsigned r0 = 0; r0 < total; r0 += 8) {
      const unsigned nb = total - r0 < 8u ? total - r0 : 8u;
      // stage rows r0 .. r0+nb-1: one cp.async.cg of 16 B per lane copies two 256 B rows
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const unsigned row = 2u * k + (lane >> 4);
        if (row < nb) {
          const unsigned src = lds_u32(s_rowsrc + 4u * (r0 + row));
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s_stage0 + 256u * row + 16u * (lane & 15u)),
                       "l"(tbase0 + src * 32u + 2u * (lane & 15u))
                       : "memory");
        }
      }
      asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
      __syncwarp();
      unsigned myS = 0, myL = 0, mySrc = 0;   // lane b keeps event b's results
#pragma unroll 1
      for (unsigned b = 0; b < nb; ++b) {
        const unsigned src = lds_u32(s_rowsrc + 4u * (r0 + b));
        unsigned long long a;
        asm volatile("ld.shared.u64 %0, [%1];" : "=l"(a) : "r"(s_stage0 + 256u * b + 8u * lane) : "memory");
        const unsigned es = __shfl_sync(FULL, E, src);
        unsigned S, L;
        sectors_lines<true, false>(a, es, lane, lanebit, lmlt, s_scr, S, L);
        const bool mine = lane == b;
        myS = mine ? S : myS;
        myL = mine ? L : myL;
        mySrc = mine ? src : mySrc;
      }
      // the batch's shared updates in one go: lanes 0..nb-1 each own one event
      const unsigned ps = __shfl_sync(FULL, pcs, mySrc);
      const bool own = lane < nb;
      red_shared_add_if(own, s_sS + 4u * ps, myS);
      red_shared_add_if(own, s_sL + 4u * ps, myL);
      red_shared_add_if(own, s_base + 4u * (6 * P + myS), 1u);        // hS[S]
      red_shared_add_if(own, s_base + 4u * (6 * P + 33 + myL), 1u);   // hL[L]
      __syncwarp();
    }
    h = hn;
  }
  red_shared_add_if(hS != 0u, s_base + 4u * (6 * P + 1 + lane), hS);
  red_shared_add_if(hL != 0u, s_base + 4u * (6 * P + 34 + lane), hL);
  bad = __reduce_add_sync(FULL, bad);
  if (lane == 0 && bad) atomicAdd(err, (unsigned long long)bad);
  __syncthreads();
  const unsigned* sA = sm;
  const unsigned* sW = sm + P;
  const unsigned* sDT = sm + 2 * P;
  const unsigned* sDW = sm + 3 * P;
  const unsigned* sS = sm + 4 * P;
  const unsigned* sL = sm + 5 * P;
  const unsigned* sH = sm + 6 * P;
  for (unsigned pc = threadIdx.x; pc < P; pc += blockDim.x) {
    const unsigned a = sA[pc], w = sW[pc];
    if (w) {
      unsigned long long* s = st.site + 4 * pc;
      atomicAdd(s + 0, (unsigned long long)a);
      atomicAdd(s + 1, (unsigned long long)(a - sDT[pc]));
      atomicAdd(s + 2, (unsigned long long)w);
      atomicAdd(s + 3, (unsigned long long)(w - sDW[pc]));
      if (sK[pc] && w != sDW[pc]) {
        unsigned long long* m = st.mem + 3 * pc;
        atomicAdd(m + 0, (unsigned long long)(w - sDW[pc]));
        atomicAdd(m + 1, (unsigned long long)sS[pc]);
        atomicAdd(m + 2, (unsigned long long)sL[pc]);
      }
    }
  }
  for (unsigned i = threadIdx.x; i < 66; i += blockDim.x)
    if (sH[i]) atomicAdd(st.hist + i, (unsigned long long)sH[i]);
}

static size_t replay4_smem(unsigned P) {
  return (((6ull * P + 66 + 3) & ~3ull) + (size_t)L4_NW * L4_WARP_WORDS) * 4 + P + 16;
}

// ---------------------------------------------------------------- staged replay (two passes per chunk)
// The single-pass kernels hold 6 x 4096 u32 per-pc bins in shared memory, which leaves little room for
// staging address slots. The staged replay splits the work along its two data streams:
//   pass A (k_rpA, 2 CTAs x 20 warps per SM): streams the 16 B headers through a per-warp cp.async ring
//     (4 tiles in flight), does items 1-3 of EM §2 (per-pc issued/executed bins, per-warp arrays) and
//     writes each executed memory event as one 8 B entry {E, pc | tile | lane} to its warp's region of a
//     caller-owned list, compacted;
//   pass B (k_rpB, 20 warps per SM): streams the listed 256 B slots into per-warp shared stages
//     (cp.async, double buffered, list entries prefetched a group ahead) and computes S/L lane-parallel:
//     two lanes per slot each scan 16 addresses, counting sector/line changes (exact when the addresses
//     of E are non-decreasing within one 4 GB region) and their min/max, so the other rows go straight
//     to the matching exact warp-cooperative path (1 KB word, 32 KB window, hashed).
// Extra traffic: 16 B per executed memory event (list write + read), ~5 % of the algorithmic bytes.
constexpr int RA_NW = 20;     // pass A warps per CTA (one list region per warp)
#ifndef NVBT_RPB_NW
#define NVBT_RPB_NW 20
#endif
constexpr int RB_NW = NVBT_RPB_NW;     // pass B warps per CTA
// Pass-B variants measured in round 2 and removed (code in commit 834b1ce; profiles/r2_replay_ab.txt, identical
// results in each): TMA tile::gather4 stages with mbarriers (r2_ab16, slower), an L2 prefetch of the next
// group (r2_ab15), global per-pc bins with 20-23 warps and dynamic regions (r2_ab19-20), two wide rows per
// iteration (r2_ab17, r2_ab25), class-0 rows by REDUX.OR (r2_ab16), an 80-register cap (r2_ab20). Kept:
// the wide-row owner resolve (r2_ab16), the multiplicative-hash bucket (r2_ab21), unpredicated per-row
// reductions and LOP3 stage offsets (r2_ab22), the row k + 8h staging (r2_ab23).
#ifndef NVBT_RPB_EXPERIMENT
#define NVBT_RPB_EXPERIMENT 0   // timing experiments (tools/replay_ab.py), never in a product build
#endif
#ifndef NVBT_RPB_SBITS
#define NVBT_RPB_SBITS 0       // 1 KB-word rows settled from sector bits gathered in the scan (A/B r2_ab10:
                               // the 2 ALU ops per address cost more than the window loop they save)
#endif
#ifndef NVBT_RPB_HIRAW
#define NVBT_RPB_HIRAW 1       // high-word check over all scanned lanes, inactive ones too (no select per
                               // address; r2_ab10: pass B 1.90 -> 1.84 ms with SBITS 0). A row whose inactive
                               // lanes differ in the upper word only takes the exact wide path.
#endif
#ifndef NVBT_RPB_WIN
#define NVBT_RPB_WIN 512       // window rows: sectors per tag window, 1024 / WIN rows per iteration (A/B r2_ab9: 256 and 128 slower)
#endif
#ifndef NVBT_RPB_TAGS
#define NVBT_RPB_TAGS 1        // slow rows by tag arrays (0: round-1 atomics + reductions, for A/B)
#endif
constexpr int RA_CTAS_PER_SM = 2;   // pass A CTAs per SM
constexpr int RA_DEPTH = 4;   // pass A header tiles in flight per warp
constexpr int RB_ROWS = 16;   // slots per stage
#ifndef NVBT_RPB_STAGES
#define NVBT_RPB_STAGES 2
#endif
constexpr int RB_STAGES = NVBT_RPB_STAGES;   // per-warp shared stages (RB_STAGES - 1 groups in flight ahead). A/B
                                             // r2_ab24: 3 stages x 13 warps 2.49 ms, 3 x 16 (global bins) 2.26, 2 x 16
                                             // 2.25, 2 x 20 1.77: the pass needs warps, not depth
// per-warp scratch, 1280 B: the slow rows' tag arrays (1 KB sector / hash tags + 256 B line tags); the
// A/B build without them (NVBT_RPB_TAGS=0) uses its first SCRATCH_WORDS words as sectors_lines_cls scratch
constexpr int RB_SCR2 = 128;
constexpr int RB_WARP_WORDS = RB_STAGES * (RB_ROWS * 64 + 2 * RB_ROWS) + SCRATCH_WORDS + RB_SCR2;
constexpr size_t RS_COUNTS_BYTES = 65536;   // u32 per pass-A warp (<= 16384 warps)
static_assert(RB_WARP_WORDS % 4 == 0, "16 B aligned warp areas");

__device__ __forceinline__ void lds_v2(unsigned a, unsigned& x, unsigned& y) {
  asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(x), "=r"(y) : "r"(a) : "memory");
}

// List entry of an executed memory event: {E, pc << 20 | k << 5 | lane}, where the event is lane `lane`
// of the k-th tile of pass-A warp r (the entry's region): event index (r + k * warps) * 32 + lane.
template <bool PW>
__global__ void __launch_bounds__(32 * RA_NW, RA_CTAS_PER_SM)
k_rpA(const uint4* __restrict__ hdr, unsigned n, unsigned P, const uint8_t* __restrict__ kind, DevState st,
      unsigned long long* err, unsigned* __restrict__ counts, uint2* __restrict__ l_ent, unsigned region_cap) {
  extern __shared__ __align__(16) unsigned sm[];
  uint8_t* sK = reinterpret_cast<uint8_t*>(sm + 4 * P);
  for (unsigned i = threadIdx.x; i < 4 * P; i += blockDim.x) sm[i] = 0;
  for (unsigned i = threadIdx.x; i < P; i += blockDim.x) sK[i] = is_mem_kind(kind[i]);
  __syncthreads();
  const unsigned lane = lane_id(), lmlt = lanemask_lt();
  const unsigned s_base = (unsigned)__cvta_generic_to_shared(sm);
  const unsigned s_kind = (unsigned)__cvta_generic_to_shared(sK);
  const unsigned gw = blockIdx.x * RA_NW + (threadIdx.x >> 5);
  const unsigned warps = gridDim.x * RA_NW;
  uint2* const ent = l_ent + (unsigned long long)gw * region_cap;
  unsigned cnt = 0, bad = 0, k = 0;
  // headers RA_DEPTH tiles ahead: per-warp ring of 512 B tile slots filled by cp.async (16 B per lane;
  // each lane reads back only what it copied, so no warp barrier is needed)
  const unsigned s_hq = s_base + 16u * P + ((P + 15u) & ~15u) + 512u * RA_DEPTH * (threadIdx.x >> 5) + 16u * lane;
#pragma unroll
  for (int d = 0; d < RA_DEPTH; ++d) {
    const unsigned i = (gw + d * warps) * 32 + lane;
    if (i < n) asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s_hq + 512u * d), "l"(hdr + i) : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
  }
  // slot d holds tile (round + d); it is refilled with tile (round + d + DEPTH) once consumed
  for (unsigned round = gw; round * 32 < n; round += RA_DEPTH * warps) {
#pragma unroll
   for (int d = 0; d < RA_DEPTH; ++d) {
    const unsigned tile = round + d * warps;
    if (tile * 32 >= n) break;
    asm volatile("cp.async.wait_group %0;" ::"n"(RA_DEPTH - 1) : "memory");
    uint4 h;
    lds_v4(s_hq + 512u * d, h);
    const unsigned i = tile * 32 + lane;
    const bool valid = i < n;
    const unsigned pc = h.x, A = h.z, E = h.z & h.w;
    const bool ok = valid && pc < P && A != 0u;
    bad += valid && pc >= P;
    const unsigned pcs = ok ? pc : 0u;
    const unsigned a4 = s_base + 4u * pcs;
    const unsigned pa = __popc(A), pe = __popc(E);
    red_shared_add_if(ok, a4, pa);
    red_shared_add_if(ok, a4 + 4u * P, 1u);
    red_shared_add_if(ok && pa != pe, a4 + 8u * P, pa - pe);
    red_shared_add_if(ok && E == 0u, a4 + 12u * P, 1u);
    if constexpr (PW) {
      const unsigned warp = h.y;
      if (ok && warp < st.n_warps) {
        atomicAdd(st.pw + warp, (unsigned long long)pe);
        if (E) atomicAdd(st.pw + st.n_warps + warp, 1ull);
      }
    }
    const bool mem = ok && E != 0u && lds_u8(s_kind + pcs) != 0u;
    const unsigned mm = __ballot_sync(FULL, mem);
    if (mem && l_ent != nullptr) ent[cnt + __popc(mm & lmlt)] = make_uint2(E, pc << 20 | k << 5 | lane);
    cnt += __popc(mm);
    ++k;
    const unsigned in = i + RA_DEPTH * warps * 32;
    if (in < n) asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s_hq + 512u * d), "l"(hdr + in) : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
   }
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  if (lane == 0 && counts != nullptr) counts[gw] = cnt;
  bad = __reduce_add_sync(FULL, bad);
  if (lane == 0 && bad) atomicAdd(err, (unsigned long long)bad);
  __syncthreads();
  const unsigned* sA = sm;
  const unsigned* sW = sm + P;
  const unsigned* sDT = sm + 2 * P;
  const unsigned* sDW = sm + 3 * P;
  for (unsigned pc = threadIdx.x; pc < P; pc += blockDim.x) {
    const unsigned a = sA[pc], w = sW[pc];
    if (w) {
      unsigned long long* s = st.site + 4 * pc;
      atomicAdd(s + 0, (unsigned long long)a);
      atomicAdd(s + 1, (unsigned long long)(a - sDT[pc]));
      atomicAdd(s + 2, (unsigned long long)w);
      atomicAdd(s + 3, (unsigned long long)(w - sDW[pc]));
      if (sK[pc] && w != sDW[pc]) atomicAdd(st.mem + 3 * pc, (unsigned long long)(w - sDW[pc]));
    }
  }
}

// c += (x > K) as a predicated add (the compiler's select-based form costs ~3 instructions)
template <unsigned K>
__device__ __forceinline__ void inc_if_gt(unsigned& c, unsigned x) {
  asm("{\n\t.reg .pred p;\n\tsetp.gt.u32 p, %1, %2;\n\t@p add.u32 %0, %0, 1;\n\t}" : "+r"(c) : "r"(x), "n"(K));
}

// Exact S, L of one row by a bitonic sort of the sector keys of its active lanes (key a >> 5 of lane `lane`).
__device__ __forceinline__ void sl_bitonic(unsigned long long a, bool act, unsigned lane, unsigned& sx, unsigned& lx) {
  unsigned long long k = act ? a >> 5 : ~0ull;
#pragma unroll
  for (unsigned kk = 2; kk <= 32; kk <<= 1) {
#pragma unroll
    for (unsigned jj = kk >> 1; jj > 0; jj >>= 1) {
      const unsigned long long o = __shfl_xor_sync(FULL, k, jj);
      const bool up = (lane & kk) == 0u, lower = (lane & jj) == 0u;
      k = (lower == up) ? (o < k ? o : k) : (o > k ? o : k);
    }
  }
  const unsigned long long pk = __shfl_up_sync(FULL, k, 1);
  const bool valid = k != ~0ull;
  sx = __popc(__ballot_sync(FULL, valid && (lane == 0u || pk != k)));
  lx = __popc(__ballot_sync(FULL, valid && (lane == 0u || (pk >> 2) != (k >> 2))));
}

// Byte offset of address idx (0..31) of stage row r. cp.async stages: row r at 256 r, 16 B chunk c at chunk
// c ^ (r & 7). TMA stages: the two 128 B halves of every row in separate 2 KB blocks (row r at 128 r), chunks
// XOR-swizzled by (r & 7) -- the tensor map's 128 B swizzle on a 1024-aligned stage.
__device__ __forceinline__ unsigned rb_off(unsigned r, unsigned idx) {
  // 8 (32 r + (idx ^ 2 (r & 7))): with a = 34 r (32 r in bits 5.., 2 r in bits 1..4), the index is
  // idx ^ (a & c) for c = ~0x11 (bits 5.. of idx are zero; bit 4 of 2 r must not flip idx): one LOP3
  unsigned x;
  asm("lop3.b32 %0, %1, %2, %3, 0x6C;" : "=r"(x) : "r"(34u * r), "r"(idx), "r"(0xFFFFFFEEu));   // b ^ (a & c)
  return 8u * x;
}

// Pass B analysis of one stage (up to 16 slots; meta E = 0 marks an empty row). Lane (j, h) = (lane & 15,
// lane >> 4) scans addresses 16h .. 16h+15 of row j; 16 B chunk c of row j is stored at chunk c ^ (j & 7),
// so the 8 lanes of a quarter-warp (consecutive j, same h) read 8 distinct bank groups.
__device__ __forceinline__ void rb_process(unsigned stage, unsigned meta, unsigned lane, unsigned lanebit,
                                           unsigned s_scr, unsigned s_sS, unsigned s_sL, unsigned s_hist) {
  const unsigned j = lane & 15u, h = lane >> 4;
  // window sectors of class 1 (tags build: kWR rows in flight, kWin + kWin / 4 tag bytes each)
  constexpr unsigned kWin = NVBT_RPB_TAGS ? NVBT_RPB_WIN : 1024u;
  constexpr int kWR = NVBT_RPB_TAGS ? 1024 / NVBT_RPB_WIN : 1;
  unsigned E, pc;
  lds_v2(meta + 8u * j, E, pc);
  const unsigned Eh = h ? E >> 16 : E & 0xffffu;
  const unsigned f = (Eh ? (unsigned)__ffs(Eh) - 1u : 0u) + 16u * h;
  unsigned f_lo, f_hi;
  lds_v2(stage + rb_off(j, f), f_lo, f_hi);
  unsigned prev = f_lo, hb = 0, bs = 0, bl = 0, mn = f_lo, mx = f_lo;
#if NVBT_RPB_TAGS && NVBT_RPB_SBITS
  unsigned sbits = 0;   // the 1 KB-word sector bits of the scanned addresses (bit (a >> 5) & 31)
#endif
  bool viol = false;
#pragma unroll
  for (int q = 0; q < ((NVBT_RPB_EXPERIMENT & 2) ? 1 : 8); ++q) {   // (experiment 2: scan 2 addresses only)
    uint4 v;
    lds_v4(stage + rb_off(j, 16u * h + 2u * q), v);
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const bool act = (Eh >> (2 * q + u)) & 1u;
      const unsigned lo = act ? (u ? v.z : v.x) : prev;
#if NVBT_RPB_HIRAW   // upper words of every scanned lane (inactive ones too: a row whose inactive lanes
      hb |= (u ? v.w : v.y) ^ f_hi;   // differ only goes to the exact wide path)
#else
      const unsigned hi = act ? (u ? v.w : v.y) : f_hi;
      hb |= hi ^ f_hi;
#endif
      viol |= lo < prev;
      const unsigned x = lo ^ prev;
      inc_if_gt<31>(bs, x);
      inc_if_gt<127>(bl, x);
      mn = min(mn, lo);
      mx = max(mx, lo);
#if NVBT_RPB_TAGS && NVBT_RPB_SBITS
      sbits |= __funnelshift_l(0u, 1u, lo >> 5);   // 1 << ((lo >> 5) & 31): one SHF.L.W
#endif
      prev = lo;
    }
  }
  // join the halves on the h = 0 lane
  const bool mine = Eh != 0u;
  const unsigned pack = bs | bl << 8 | (unsigned)viol << 16 | (unsigned)(hb != 0u) << 17 | (unsigned)mine << 18;
  const unsigned o_pack = __shfl_xor_sync(FULL, pack, 16);
  const unsigned o_lo = __shfl_xor_sync(FULL, f_lo, 16);
  const unsigned o_hi = __shfl_xor_sync(FULL, f_hi, 16);
  const unsigned o_mn = __shfl_xor_sync(FULL, mn, 16);
  const unsigned o_mx = __shfl_xor_sync(FULL, mx, 16);
#if NVBT_RPB_TAGS && NVBT_RPB_SBITS
  const unsigned o_sb = __shfl_xor_sync(FULL, sbits, 16);
#endif
  const bool other = (o_pack >> 18) != 0u;
  unsigned S = 1u + bs + (o_pack & 0xffu), L = 1u + bl + ((o_pack >> 8) & 0xffu);
  bool hb_row = hb != 0u || ((o_pack >> 17) & 1u) != 0u;
  bool slow = viol || ((o_pack >> 16) & 1u) != 0u;
  if (mine && other) {
    const unsigned x = o_lo ^ prev;
    S += x > 31u;
    L += x > 127u;
    slow |= o_lo < prev;
    hb_row |= o_hi != f_hi;
  }
  slow |= hb_row;
  const unsigned rmn = mine ? (other ? min(mn, o_mn) : mn) : o_mn;
  const unsigned rmx = mine ? (other ? max(mx, o_mx) : mx) : o_mx;
  const unsigned wbase = (rmn >> 5) & ~31u;
  // classes: 0 = one 1 KB word, 1 = a window of kWin sectors from wbase, 2 = anything else
  const unsigned cls = hb_row ? 2u : (rmn >> 10) == (rmx >> 10) ? 0u : ((rmx >> 5) - wbase < kWin ? 1u : 2u);
  const bool own = h == 0u && E != 0u;
  // rows that are not monotone within one 4 GB region: exact paths, one loop per class of the row's
  // address range (one 1 KB word / a 32 KB window / anything else)
  // (NVBT_RPB_EXPERIMENT bits 1, 4, 8, 16: timing experiments only, wrong results: drop all / class-0 /
  // class-1 / class-2 slow rows)
#if NVBT_RPB_TAGS && NVBT_RPB_SBITS
  if (slow && cls == 0u) {   // one 1 KB word: the scan's sector bits are exact (no loop below)
    const unsigned word = (mine ? sbits : 0u) | (other ? o_sb : 0u);
    const unsigned g = word | (word >> 1) | (word >> 2) | (word >> 3);
    S = __popc(word);
    L = __popc(g & 0x11111111u);
  }
  const unsigned cm0 = 0u;
#elif NVBT_RPB_TAGS
  const unsigned cm0 = (NVBT_RPB_EXPERIMENT & 5) ? 0u : __ballot_sync(FULL, own && slow && cls == 0u);   // window loop takes class 0 too
#else
  const unsigned cm0 = (NVBT_RPB_EXPERIMENT & 5) ? 0u : __ballot_sync(FULL, own && slow && cls == 0u);
#endif
  const unsigned cm1 = (NVBT_RPB_EXPERIMENT & 9) ? 0u : __ballot_sync(FULL, own && slow && cls == 1u);
  const unsigned cm2 = (NVBT_RPB_EXPERIMENT & 17) ? 0u : __ballot_sync(FULL, own && slow && cls == 2u);
#if NVBT_RPB_TAGS
  // Exact distinct counts without atomics or reductions: every active lane stores its lane id (u8) at its
  // key's slot of a per-warp tag array and reads the slot back after a __syncwarp; of the lanes sharing a
  // slot exactly one (the last writer) reads its own id, so the number of distinct slots = popc(ballot(own
  // id read)). Stale tags from earlier rows never matter: every lane that reads a slot wrote it this row.
  //  * rows within one 1 KB word (class 0) are settled from the scan's sector bits above;
  //  * window rows (all sectors of E in the kWin-sector window from wbase, upper words equal; class 1):
  //    the slot is the sector's offset in the window (kWin tag bytes) and, for lines, offset >> 2: S and L
  //    exactly; 1024 / kWin rows per iteration;
  //  * wide rows (class 2): all lines distinct? slots = a hash of the line into 1280 buckets; all lanes
  //    owning their slot proves every line (hence sector) distinct: S = L = |E|; collisions are resolved
  //    against the bucket owners (below). Rows with a three-way collision or a repeated line (~0.3 %) take
  //    an exact bitonic sort of the sector keys.
  const unsigned stag = s_scr, ltag = s_scr + 1024u;
  unsigned mw = cm0 | cm1, mwide = cm2;
  // up to kWR window rows per iteration (independent chains; per row a kWin-sector window of tags and
  // kWin / 4 line tags)
  while (mw) {
    unsigned r[kWR], lo[kWR], off[kWR], ev[kWR], wv[kWR];
    bool v[kWR], act[kWR];
#pragma unroll
    for (int k = 0; k < kWR; ++k) {
      v[k] = mw != 0u;
      r[k] = v[k] ? 31u - __clz(mw) : 0u;
      if (v[k]) mw ^= 1u << r[k];
    }
#pragma unroll
    for (int k = 0; k < kWR; ++k) {
      ev[k] = __shfl_sync(FULL, E, r[k]);
      wv[k] = __shfl_sync(FULL, wbase, r[k]);
      lo[k] = lds_u32(stage + rb_off(r[k], lane));
    }
#pragma unroll
    for (int k = 0; k < kWR; ++k) {
      act[k] = v[k] && ((ev[k] >> lane) & 1u);
      off[k] = (lo[k] >> 5) - wv[k];
      if (act[k]) {
        sts_u8(stag + kWin * k + off[k], lane);
        sts_u8(ltag + (kWin / 4u) * k + (off[k] >> 2), lane);
      }
    }
    __syncwarp();
#pragma unroll
    for (int k = 0; k < kWR; ++k) {
      const bool fs = act[k] && lds_u8(stag + kWin * k + off[k]) == lane;
      const bool fl = act[k] && lds_u8(ltag + (kWin / 4u) * k + (off[k] >> 2)) == lane;
      const unsigned sx = __popc(__ballot_sync(FULL, fs)), lx = __popc(__ballot_sync(FULL, fl));
      S = (v[k] && lane == r[k]) ? sx : S;
      L = (v[k] && lane == r[k]) ? lx : L;
    }
    __syncwarp();                                  // reads done before the next rows' stores
  }
  while (mwide) {
    const unsigned src = 31u - __clz(mwide);
    mwide ^= 1u << src;
    const unsigned es = __shfl_sync(FULL, E, src);
    unsigned long long a;
    asm volatile("ld.shared.u64 %0, [%1];" : "=l"(a) : "r"(stage + rb_off(src, lane)) : "memory");
    const bool act = (es >> lane) & 1u;
    const unsigned long long line = a >> 7;
    const unsigned x0 = (unsigned)line, x1 = (unsigned)(line >> 32);
    bool ok;
    {
      // one hash round; if a lane lost its bucket, every loser compares its line with the bucket's owner (the
      // last writer) and the losers tag their buckets again: when each loser then owns its bucket, every
      // bucket holds the owner and at most one loser whose line differs from the owner's, so all lines are
      // distinct (equal lines always share a bucket). Anything else takes the exact sort below.
      const unsigned hsh = x0 * 0x9E3779B1u ^ x1 * 0x85EBCA77u;
      const unsigned hb = __umulhi(hsh, 1280u);   // Fibonacci hashing: the product's top bits
      if (act) sts_u8(stag + hb, lane);
      __syncwarp();
      const unsigned own = lds_u8(stag + hb) & 31u;
      const bool lose = act && own != lane;
      ok = !__any_sync(FULL, lose);
      if (!ok) {                                   // warp-uniform
        const unsigned o0 = __shfl_sync(FULL, x0, own), o1 = __shfl_sync(FULL, x1, own);
        const bool same = lose && o0 == x0 && o1 == x1;
        if (lose) sts_u8(stag + hb, lane);         // every lane has read its owner (__any_sync above)
        __syncwarp();
        const bool lose2 = lose && lds_u8(stag + hb) != lane;
        ok = !__any_sync(FULL, same || lose2);
      }
      __syncwarp();
    }
    unsigned sx, lx;
    if (ok) {
      sx = lx = __popc(es);
    } else {                                       // exact: bitonic sort of the sector keys of E
      sl_bitonic(a, act, lane, sx, lx);
    }
    S = lane == src ? sx : S;
    L = lane == src ? lx : L;
  }
#else
  // one row per iteration, warp-cooperative; lane l reads address l
  unsigned m0 = cm0, m1 = cm1, m2 = cm2;
  const unsigned l8 = 8u * lane;
  while (m0) {
    const unsigned src = 31u - __clz(m0);
    m0 ^= 1u << src;
    const unsigned es = __shfl_sync(FULL, E, src);
    const unsigned a_lo = lds_u32(stage + rb_off(src, lane));
    const uint2 r = sl_word(a_lo, (es & lanebit) != 0u);
    S = lane == src ? r.x : S;
    L = lane == src ? r.y : L;
  }
  while (m1) {
    const unsigned src = 31u - __clz(m1);
    m1 ^= 1u << src;
    const unsigned es = __shfl_sync(FULL, E, src), wb = __shfl_sync(FULL, wbase, src);
    const unsigned a_lo = lds_u32(stage + rb_off(src, lane));
    const uint2 r = sl_window(a_lo, (es & lanebit) != 0u, lane, s_scr, wb);
    S = lane == src ? r.x : S;
    L = lane == src ? r.y : L;
  }
  while (m2) {
    const unsigned src = 31u - __clz(m2);
    m2 ^= 1u << src;
    const unsigned es = __shfl_sync(FULL, E, src);
    unsigned long long a;
    asm volatile("ld.shared.u64 %0, [%1];" : "=l"(a) : "r"(stage + rb_off(src, lane)) : "memory");
    const uint2 r = sl_wide(a, es, lanebit, lane, s_scr);
    S = lane == src ? r.x : S;
    L = lane == src ? r.y : L;
  }
#endif
  {
    const unsigned dmy = s_scr + 4u * lane;   // lane-private word: adding 0 changes nothing
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(own ? s_sS + 4u * pc : dmy), "r"(own ? S : 0u) : "memory");
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(own ? s_sL + 4u * pc : dmy), "r"(own ? L : 0u) : "memory");
  }
  {
    const unsigned dmy = s_scr + 4u * lane, one = own ? 1u : 0u;
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(own ? s_hist + 4u * S : dmy), "r"(one) : "memory");          // hS[S]
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(own ? s_hist + 4u * (33u + L) : dmy), "r"(one) : "memory");  // hL[L]
  }
  __syncwarp();
}

__global__ void __launch_bounds__(32 * RB_NW, 1)
k_rpB(const unsigned long long* __restrict__ addr, unsigned P, const uint8_t* __restrict__ kind, DevState st,
      const unsigned* __restrict__ counts, unsigned n_regions, const uint2* __restrict__ l_ent, unsigned region_cap) {
  extern __shared__ __align__(16) unsigned sm[];
  const unsigned PB = (2 * P + 66 + 3) & ~3u;      // sS[P] | sL[P] | hist[66]
  for (unsigned i = threadIdx.x; i < PB; i += blockDim.x) sm[i] = 0;
  const unsigned lane = lane_id(), lanebit = 1u << lane;
  const unsigned s_base = (unsigned)__cvta_generic_to_shared(sm);
  // warp areas 128-byte aligned (9728 B each): stage chunk offsets can then be XOR-ed into full addresses
  unsigned* sWarpAll = reinterpret_cast<unsigned*>((reinterpret_cast<uintptr_t>(sm + PB) + 127u) & ~uintptr_t(127));
  static_assert((RB_WARP_WORDS * 4) % 128 == 0, "128 B aligned warp areas");
  constexpr unsigned kScr0 = RB_STAGES * (RB_ROWS * 64 + 2 * RB_ROWS);
  for (unsigned i = threadIdx.x; i < RB_NW * RB_WARP_WORDS; i += blockDim.x) {
    const unsigned o = i % RB_WARP_WORDS;
    sWarpAll[i] = o >= kScr0 + SCRATCH_WORDS ? 0xffffffffu : o >= kScr0 ? scratch_init_word(o - kScr0) : 0u;
  }
  __syncthreads();
  const unsigned s_w = (unsigned)__cvta_generic_to_shared(sWarpAll + (threadIdx.x >> 5) * RB_WARP_WORDS);
  const unsigned s_meta = s_w + 4u * RB_STAGES * RB_ROWS * 64;      // stage s: + 128 s
  const unsigned s_scr = s_w + 4u * kScr0;
  const unsigned s_sS = s_base, s_sL = s_base + 4u * P, s_hist = s_base + 8u * P;
  const unsigned WB = gridDim.x * RB_NW;
  const unsigned j = lane & 15u, h = lane >> 4;
  // group cursor over this warp's regions gw, gw + WB, ...
  unsigned r = blockIdx.x * RB_NW + (threadIdx.x >> 5), off = 0;
  unsigned rcnt = r < n_regions ? counts[r] : 0u;
  // a group: up to 16 list entries of one region (row j in lanes j and j + 16), loaded ahead of use
  struct Grp { unsigned rows, r; uint2 ent; };
  auto fetch = [&](Grp& g) {
    while (r < n_regions && off >= rcnt) {
      r += WB;
      off = 0;
      rcnt = r < n_regions ? counts[r] : 0u;
    }
    g.rows = r < n_regions ? min(rcnt - off, (unsigned)RB_ROWS) : 0u;
    const unsigned long long p = (unsigned long long)r * region_cap + off + j;
    g.ent = j < g.rows ? l_ent[p] : make_uint2(0u, 0u);   // decoded at use (load in flight)
    g.r = r;
    off += g.rows;
  };
  auto slot_of = [&](const Grp& g) -> unsigned {   // event index of row j's slot
    return (g.r + ((g.ent.y >> 5) & 0x7fffu) * n_regions) * 32u + (g.ent.y & 31u);
  };
  Grp g1{};   // the next group to stage
  // stage g1 into stage s (meta + slot copies), then fetch the next group
  auto issue = [&](unsigned s) {
    const unsigned nx_E = g1.ent.x, nx_pc = g1.ent.y >> 20;
    const unsigned nx_idx = slot_of(g1);
    if (h == 0u)
      asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(s_meta + 128u * s + 8u * j), "r"(nx_E), "r"(nx_pc) : "memory");
    const unsigned stg = s_w + 4096u * s;
    // step k: lane (h, c) copies 16 B chunk c of row k + 8h. Row r's chunk c lives at 256 r + 16 (c ^ (r & 7)) =
    // 256 k + (lane_off ^ 16 k) with lane_off = 2048 h + 16 c (r & 7 == k). The upper half first takes the slot
    // indices of rows 8..15, so step k's index comes from source lane k of each half (width-16 shuffle).
    const unsigned idx_st = __shfl_sync(FULL, nx_idx, h ? ((lane + 8u) & 15u) : lane);
    const unsigned sb = stg + 2048u * h + 16u * (lane & 15u);   // stg is 128-aligned: XOR 16 k stays in the chunk bits
    const unsigned long long* gl = addr + 2u * (lane & 15u);
    if (g1.rows == (unsigned)RB_ROWS) {            // warp-uniform: a full group
#pragma unroll
      for (int k = 0; k < RB_ROWS / 2; ++k) {
        const unsigned ix = __shfl_sync(FULL, idx_st, k, 16);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                     ::"r"((sb ^ (16u * k)) + 256u * k), "l"(gl + (unsigned long long)ix * 32u) : "memory");
      }
    } else {
#pragma unroll
      for (int k = 0; k < RB_ROWS / 2; ++k) {
        const unsigned ix = __shfl_sync(FULL, idx_st, k, 16);
        if ((unsigned)k + 8u * h < g1.rows)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                       ::"r"((sb ^ (16u * k)) + 256u * k), "l"(gl + (unsigned long long)ix * 32u) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    fetch(g1);
  };
  fetch(g1);
  // RB_STAGES - 1 groups in flight ahead of the one being analysed; stage (s + RB_STAGES - 1) % RB_STAGES was
  // analysed in the previous step. Steps without a group to issue commit an empty cp.async group, so
  // wait_group(RB_STAGES - 1) always retires the oldest issued one.
  unsigned s = 0, pending = 0;
#pragma unroll
  for (int i = 0; i < RB_STAGES - 1; ++i) {
    if (g1.rows != 0u) { issue((unsigned)i); ++pending; }
    else asm volatile("cp.async.commit_group;" ::: "memory");
  }
  while (pending) {
    const unsigned sn = s == 0u ? (unsigned)RB_STAGES - 1u : s - 1u;
    if (g1.rows != 0u) { issue(sn); ++pending; }
    else asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_group %0;" ::"n"(RB_STAGES - 1) : "memory");
    __syncwarp();
    rb_process(s_w + 4096u * s, s_meta + 128u * s, lane, lanebit, s_scr, s_sS, s_sL, s_hist);
    --pending;
    s = s + 1u == (unsigned)RB_STAGES ? 0u : s + 1u;
  }
  __syncthreads();
  const uint8_t* kd = kind;
  for (unsigned pc = threadIdx.x; pc < P; pc += blockDim.x) {
    const unsigned a = sm[pc], b = sm[P + pc];
    if (is_mem_kind(kd[pc]) && (a | b)) {
      atomicAdd(st.mem + 3 * pc + 1, (unsigned long long)a);
      atomicAdd(st.mem + 3 * pc + 2, (unsigned long long)b);
    }
  }
  for (unsigned i = threadIdx.x; i < 66; i += blockDim.x)
    if (sm[2 * P + i]) atomicAdd(st.hist + i, (unsigned long long)sm[2 * P + i]);
}

static size_t rpA_smem(unsigned P) { return 16ull * P + ((P + 15ull) & ~15ull) + 512ull * RA_DEPTH * RA_NW; }
static size_t rpB_smem(unsigned P) {
  return (((2ull * P + 66 + 3) & ~3ull) + (size_t)RB_NW * RB_WARP_WORDS) * 4 + 128;
}

static int sm_count(int dev) { return device_sms(dev); }


}  // namespace nvbt

using namespace nvbt;

extern "C" {

int nvbt_program(int w, nvbt_instr_desc* out, uint32_t cap, uint32_t* n_pcs, uint32_t* n_ops, uint32_t* n_bbs) {
  const nvbt_instr_desc* t = nullptr;
  uint32_t n = 0, o = kWorkloadOpcodes, b = 0;
  static nvbt_instr_desc replay_prog[4096];
  static bool replay_built = false;
  switch (w) {
    case NVBT_W_VECTORADD: t = ProgVectorAdd::t; n = ProgVectorAdd::N; break;
    case NVBT_W_SGEMM: t = ProgSgemm::t; n = ProgSgemm::N; break;
    case NVBT_W_BFS: t = ProgBfs::t; n = ProgBfs::N; break;
    case NVBT_W_STENCIL: t = ProgStencil::t; n = ProgStencil::N; break;
    case NVBT_W_WFFT_EMU: t = ProgWfftEmu::t; n = ProgWfftEmu::N; o = kWfftOpcodes; break;
    case NVBT_W_WFFT_SW: t = ProgWfftSw::t; n = ProgWfftSw::N; o = kWfftOpcodes; break;
    case NVBT_W_REPLAY:
      if (!replay_built) {  // EM §3.5, always from the constant SEED
        const unsigned long long k100 = Kf(kSeed, 100);
        for (uint32_t pc = 0; pc < 4096; ++pc) {
          const unsigned long long h = mix64(k100 ^ pc);
          nvbt_instr_desc d{};
          d.bb = pc >> 3;
          d.is_leader = (pc & 7) == 0;
          d.guarded = 1;
          if (h % 4 == 0) {
            d.kind = ((h >> 8) & 1) ? NVBT_K_GST : NVBT_K_GLD;
            d.width = (uint8_t)(4u << ((h >> 16) % 3));
            d.opcode = d.kind == NVBT_K_GLD ? 0 : 1;
          } else {
            d.kind = (pc & 7) == 7 ? NVBT_K_CTRL : NVBT_K_ALU;
            d.width = 0;
            d.opcode = (uint16_t)(2 + (h >> 24) % 62);
          }
          replay_prog[pc] = d;
        }
        replay_built = true;
      }
      t = replay_prog; n = 4096; o = 64;
      break;
    default: return set_error(NVBT_EINVAL, "unknown workload %d", w);
  }
  for (uint32_t i = 0; i < n; ++i) b = t[i].bb + 1 > b ? t[i].bb + 1 : b;
  if (n_pcs) *n_pcs = n;
  if (n_ops) *n_ops = o;
  if (n_bbs) *n_bbs = b;
  if (out) {
    if (cap < n) return set_error(NVBT_EINVAL, "program has %u pcs, cap %u", n, cap);
    std::memcpy(out, t, sizeof(nvbt_instr_desc) * n);
  }
  return NVBT_OK;
}

int nvbt_gen_events(nvbt_ctx c, uint64_t seed, uint64_t first, uint64_t n, void* d_hdr, void* d_addr) {
  if (!c || !d_hdr || !d_addr) return set_error(NVBT_EINVAL, "null argument");
  if ((reinterpret_cast<uintptr_t>(d_hdr) | reinterpret_cast<uintptr_t>(d_addr)) % 16)
    return set_error(NVBT_EINVAL, "stream buffers must be 16-byte aligned");
  nvbt_instr_desc prog[4096];
  uint32_t np = 0;
  int rc = nvbt_program(NVBT_W_REPLAY, prog, 4096, &np, nullptr, nullptr);
  if (rc) return rc;
  rc = check_program(c, prog, (int)np, "replay");
  if (rc) return rc;
  if (n == 0) return NVBT_OK;
  NVBT_CUDA(cudaSetDevice(c->device));
  GenConsts G;
  G.seed = seed;
  for (int f = 0; f < 9; ++f) G.k[f] = Kf(seed, f);
  const unsigned long long tiles = (n + 31) / 32;
  const int blocks = (int)std::min<unsigned long long>((tiles + 7) / 8, (unsigned long long)sm_count(c->device) * 8);
  k_gen<<<blocks, 256, 0, c->stream>>>(G, first, n, c->d_kind, c->d_prog, static_cast<uint4*>(d_hdr),
                                       static_cast<unsigned long long*>(d_addr));
  NVBT_CUDA(cudaGetLastError());
  c->launches++;
  return NVBT_OK;
}

}  // extern "C"

static int launch_replay4(nvbt_ctx c, const void* d_hdr, const void* d_addr, uint64_t n, const DevState& st) {
  const size_t smem = replay4_smem(c->n_pcs);
  int rc = func_smem((const void*)k_replay4<false>, c->device, replay4_smem(4096));
  if (!rc) rc = func_smem((const void*)k_replay4<true>, c->device, replay4_smem(4096));
  if (rc) return rc;
  const unsigned long long kMaxPerLaunch = 1ull << 30;
  const int sms = sm_count(c->device);
  for (uint64_t off = 0; off < n; off += kMaxPerLaunch) {
    const uint64_t m = std::min<uint64_t>(kMaxPerLaunch, n - off);
    const unsigned long long tiles = (m + 31) / 32;
    const int blocks = (int)std::min<unsigned long long>((tiles + 2 * L4_NW - 1) / (2 * L4_NW), (unsigned long long)sms);
    auto kern = st.pw != nullptr ? k_replay4<true> : k_replay4<false>;
    kern<<<blocks, 32 * L4_NW, smem, c->stream>>>(static_cast<const uint4*>(d_hdr) + off,
                                                  static_cast<const unsigned long long*>(d_addr) + off * 32, m,
                                                  c->n_pcs, c->d_kind, st, c->ctl + CTL_REPLAY_ERR);
    NVBT_CUDA(cudaGetLastError());
    c->launches++;
  }
  return NVBT_OK;
}

// Staged replay: scratch = counts [16384 u32] | entries [cap] (uint2, k_rpA); passes of at most
// cap - 32 * (pass-A warps) events (every pass-A warp owns a region of 32 * ceil(tiles / warps) entries).
static unsigned long long staged_cap(size_t bytes) {
  return bytes > RS_COUNTS_BYTES ? ((bytes - RS_COUNTS_BYTES) / 8) & ~63ull : 0ull;
}

static int launch_staged(nvbt_ctx c, const void* d_hdr, const void* d_addr, uint64_t n, const DevState& st,
                         void* scratch, size_t scratch_bytes) {
  int arc = func_smem((const void*)k_rpA<false>, c->device, rpA_smem(4096));
  if (!arc) arc = func_smem((const void*)k_rpA<true>, c->device, rpA_smem(4096));
  if (!arc) arc = func_smem((const void*)k_rpB, c->device, rpB_smem(4096));
  if (arc) return arc;
  const int sms = sm_count(c->device);
  const bool memdiv = (c->flags & NVBT_MEMDIV) != 0;
  const unsigned long long cap = staged_cap(scratch_bytes);
  const unsigned long long max_warps = (unsigned long long)sms * RA_CTAS_PER_SM * RA_NW;
  unsigned long long pass = 1ull << 30;   // keeps every CTA's u32 bins far from overflow
  if (max_warps > RS_COUNTS_BYTES / 4) return set_error(NVBT_EINVAL, "staged replay: %llu pass-A warps", max_warps);
  if (memdiv) {
    if (scratch == nullptr || cap <= 32ull * max_warps)
      return set_error(NVBT_ENOMEM, "staged replay scratch of %zu bytes is too small", scratch_bytes);
    if (reinterpret_cast<uintptr_t>(scratch) % 256) return set_error(NVBT_EINVAL, "scratch not 256-byte aligned");
    pass = std::min(pass, (cap - 32ull * max_warps) & ~31ull);
  }
  unsigned* counts = static_cast<unsigned*>(scratch);
  uint2* l_ent = memdiv ? reinterpret_cast<uint2*>(static_cast<char*>(scratch) + RS_COUNTS_BYTES) : nullptr;
  for (uint64_t off = 0; off < n; off += pass) {
    const uint64_t m = std::min<uint64_t>(pass, n - off);
    const unsigned long long tiles = (m + 31) / 32;
    // pass A: up to RA_CTAS_PER_SM CTAs per SM (its shared footprint allows 2), pass B: one per SM; a
    // pass-B warp takes the regions gw, gw + warps_B, ... (exactly RA_CTAS_PER_SM each on full grids)
    const int blocks = (int)std::min<unsigned long long>((tiles + 2 * RA_NW - 1) / (2 * RA_NW),
                                                         (unsigned long long)sms * RA_CTAS_PER_SM);
    const int blocks_b = std::min(blocks, sms);
    const unsigned warps = (unsigned)blocks * RA_NW;
    const unsigned region_cap = (unsigned)(32 * ((tiles + warps - 1) / warps));
    // list keys hold the tile ordinal within a warp in 15 bits (pass <= 2^30 events on >= 1024 warps, or
    // fewer events on small grids)
    if (region_cap / 32 > 32768u) return set_error(NVBT_EINVAL, "staged replay: %u tiles per warp", region_cap / 32);
    auto ka = st.pw != nullptr ? k_rpA<true> : k_rpA<false>;
    ka<<<blocks, 32 * RA_NW, rpA_smem(c->n_pcs), c->stream>>>(
        static_cast<const uint4*>(d_hdr) + off, (unsigned)m, c->n_pcs, c->d_kind, st, c->ctl + CTL_REPLAY_ERR,
        memdiv ? counts : nullptr, l_ent, region_cap);
    NVBT_CUDA(cudaGetLastError());
    c->launches++;
    if (!memdiv) continue;
    k_rpB<<<blocks_b, 32 * RB_NW, rpB_smem(c->n_pcs), c->stream>>>(
        static_cast<const unsigned long long*>(d_addr) + off * 32, c->n_pcs, c->d_kind, st, counts, warps, l_ent,
        region_cap);
    NVBT_CUDA(cudaGetLastError());
    c->launches++;
  }
  return NVBT_OK;
}

extern "C" {

int nvbt_replay_scratch_size(nvbt_ctx c, uint64_t max_events, size_t* bytes) {
  if (!c || !bytes) return set_error(NVBT_EINVAL, "null argument");
  const unsigned long long per = std::min<unsigned long long>(std::max<uint64_t>(max_events, 1), 1ull << 30);
  const unsigned long long cap = ((per + 31) & ~31ull) + 32ull * sm_count(c->device) * RA_CTAS_PER_SM * RA_NW + 64;
  *bytes = RS_COUNTS_BYTES + 8 * cap;
  return NVBT_OK;
}

int nvbt_replay_staged(nvbt_ctx c, const void* d_hdr, const void* d_addr, uint64_t n, void* d_scratch,
                       size_t scratch_bytes) {
  if (!c || !d_hdr || !d_addr) return set_error(NVBT_EINVAL, "null argument");
  if ((reinterpret_cast<uintptr_t>(d_hdr) | reinterpret_cast<uintptr_t>(d_addr)) % 16)
    return set_error(NVBT_EINVAL, "stream buffers must be 16-byte aligned");
  if (!(c->flags & (NVBT_COUNT | NVBT_OPHIST | NVBT_BB))) return set_error(NVBT_ESTATE, "replay needs NVBT_COUNT");
  DevState st;
  int rc = make_state(c, NVBT_TOOL_COUNT | ((c->flags & NVBT_MEMDIV) ? NVBT_TOOL_MEMDIV : 0), &st);
  if (rc) return rc;
  if (n == 0) return NVBT_OK;
  NVBT_CUDA(cudaSetDevice(c->device));
  return launch_staged(c, d_hdr, d_addr, n, st, d_scratch, scratch_bytes);
}

int nvbt_replay(nvbt_ctx c, const void* d_hdr, const void* d_addr, uint64_t n) {
  if (!c || !d_hdr || !d_addr) return set_error(NVBT_EINVAL, "null argument");
  if ((reinterpret_cast<uintptr_t>(d_hdr) | reinterpret_cast<uintptr_t>(d_addr)) % 16)
    return set_error(NVBT_EINVAL, "stream buffers must be 16-byte aligned");
  if (!(c->flags & (NVBT_COUNT | NVBT_OPHIST | NVBT_BB))) return set_error(NVBT_ESTATE, "replay needs NVBT_COUNT");
  DevState st;
  int rc = make_state(c, NVBT_TOOL_COUNT | ((c->flags & NVBT_MEMDIV) ? NVBT_TOOL_MEMDIV : 0), &st);
  if (rc) return rc;
  if (n == 0) return NVBT_OK;
  NVBT_CUDA(cudaSetDevice(c->device));
  return launch_replay4(c, d_hdr, d_addr, n, st);
}

}  // extern "C"
