// nvbt device hook library (L0): the compiled-in analogue of NVBit's injected device functions.
//
// NVBit injects a call before an instruction and passes it the guard predicate, register values and
// immediates (nvbit_insert_call / nvbit_add_call_arg, P:L123 (§4), P:L243-246 (§6.1)); "every active
// thread enters, then leaves, the instrumentation function" (P:L307 (§7)) after a per-thread register
// save. Here the hook is inlined at the injection point and works at warp level:
//   * event formation (a1): A = ballot(in_flow), P = ballot(in_flow && pred), E = A & P — the
//     "predicate matching before jumping" the paper proposes; one vote per mask.
//   * counting (a2-a4): per-site warp-uniform counters live in REGISTERS for the whole warp (indices are
//     compile-time pcs), i.e. the "warp-level reductions" and "radix-tree of counters, one per thread
//     block" of P:L89: registers -> CTA shared-memory bins -> one global 64-bit atomic per non-zero bin
//     per CTA (a8). Opcode/BB histograms are folded from per-pc bins at read time (fold kernel), which
//     is the same integer sum regrouped (EM §2 items 2-3).
//   * memory divergence (a5): S and L by __match_any_sync on addr>>5 / addr>>7 and a ballot of group
//     leaders (Listing 8, readings R-2..R-8): exact integer distinct counts instead of the
//     listing's float 1/cnt sum (R-5).
//   * trace (a6): one 288 B record per executed global-memory event, written by the warp straight into
//     the pinned host ring (coalesced 8 B/lane stores), committed with a tag after a system fence.
// Precondition ("converged-hook discipline"): every hook is called by all 32 lanes of the warp
// (lanes that have exited or are on another path pass in_flow = false).
#pragma once
#include <type_traits>
#include <cstdint>
#include "nvbt.h"
#include "nvbt_dev.cuh"   // public device primitives (event formation helpers, sectors_lines)

namespace nvbt {

constexpr uint32_t TOOL_COUNT = NVBT_TOOL_COUNT, TOOL_BB = NVBT_TOOL_BBCOUNT, TOOL_MEM = NVBT_TOOL_MEMDIV,
                   TOOL_TRACE = NVBT_TOOL_TRACE;
constexpr int RECORD_BYTES = 288;
// internal tool bit (not in the ABI): TRACE into a device-memory ring (F2), chosen at launch time when the
// context's channel lives in HBM, so the producer's path is selected at compile time
constexpr uint32_t TOOL_TRACE_DEV = 1u << 8;
constexpr int SITE_WORDS = 7;  // per-pc shared bins: tA, dT, wI, dW, mN, mS, mL

// POD handed by value to every instrumented kernel (kernel parameter space).
struct DevState {
  unsigned long long* site;        // [n_pcs][4] u64: t_issued, t_exec, w_issued, w_exec
  unsigned long long* mem;         // [n_pcs][3] u64: n, ΣS, ΣL
  unsigned long long* hist;        // [2][33] u64: hS, hL
  unsigned long long* pw;          // [2][n_warps] u64 or nullptr
  unsigned char* ring;             // record slots (device view of pinned host memory) or nullptr
  unsigned long long* head;        // tickets handed out (device memory)
  const unsigned long long* tail;  // records consumed by the host (device view of pinned memory)
  unsigned long long* tail_cache;  // last tail a producer saw (device memory)
  unsigned long long* dropped;     // records given up on (device memory)
  unsigned long long cap;          // ring slots
  unsigned* tags;                  // host ring: commit tag of slot i, in a dense array after the slots
  unsigned launch;
  unsigned n_warps;
  unsigned stripes;                // site/mem/hist repeat `stripes` times, stride stripe_words
  unsigned long long stripe_words;
  unsigned slot_bytes;             // slot stride: 288, 192 (176 B compact slots, EM §5.1, padded) or 128 (EM §5.2)
  unsigned compact;                // 0 full records; 1 / 2 176 B slots (2: force wide pairs); 3 / 4 128 B slots
                                   // (4: force the three-slot form)
  unsigned no_wait;                // device-memory ring (F2): drop when full instead of waiting
  unsigned long long wait_ns;      // host ring: a producer waiting this long for room gives up (drops)
  // device ring (F2): slots are handed out in chunks of kRingChunk. Each SM owns a stripe word
  // rheads[smid % rstripes] = (chunk << 32 | used) and takes tickets from its current chunk; the warp whose
  // ticket is exactly kRingChunk opens the stripe's next chunk from the global counter rheads[rstripes].
  unsigned long long* rheads;
  unsigned rstripes;
  // multi-GPU partition (nvbt_set_partition): this launch runs the CTA rows from cta_y0 on; its logical
  // linear CTA id is cta_lo + blockIdx.x + blockIdx.y * gridDim.x (cta_lo = cta_y0 * CTA-grid width)
  unsigned cta_lo;
  unsigned cta_y0;
  // launches whose loop trip counts could wrap a u32 CTA bin (BFS warps with a vertex of degree >= 2^24)
  // count themselves here; the next read call reports NVBT_EINVAL instead of wrapped results
  unsigned long long* ovf;
};
constexpr unsigned kRingChunk = 4096;
constexpr unsigned kRingNoChunk = 0xFFFFFFFEu, kRingFull = 0xFFFFFFFFu;


template <class Prog> __host__ __device__ constexpr int leader_of(int pc) {
  int p = pc;
  while (p > 0 && !Prog::t[p].is_leader) --p;
  return p;
}
template <class Prog> __host__ __device__ constexpr int bb_len(int lead) {
  int n = 1;
  while (lead + n < Prog::N && !Prog::t[lead + n].is_leader) ++n;
  return n;
}
// memory pcs in [pc, end of pc's basic block]
template <class Prog> __host__ __device__ constexpr int mem_left(int pc) {
  int n = 0;
  for (int p = pc; p < Prog::N && (p == pc || !Prog::t[p].is_leader); ++p) n += is_mem_kind(Prog::t[p].kind) ? 1 : 0;
  return n;
}
// tickets a warp reserves at memory pc `pc` (the rest of its basic block, x4 in register-mode loops)
template <class Prog> __host__ __device__ constexpr unsigned block_at(int pc) {
  return (unsigned)mem_left<Prog>(pc) * ((pc >= Prog::REG_LO && pc <= Prog::REG_HI) ? 4u : 1u);
}
template <class Prog> __host__ __device__ constexpr unsigned max_block() {
  unsigned m = 1;
  for (int p = 0; p < Prog::N; ++p) m = block_at<Prog>(p) > m ? block_at<Prog>(p) : m;
  return m;
}

// programs may opt out of 288 B trace staging (static constexpr bool kStageTrace = false)
template <class P, class = void> struct stage_trace { static constexpr bool value = true; };
template <class P> struct stage_trace<P, std::void_t<decltype(P::kStageTrace)>> { static constexpr bool value = P::kStageTrace; };

#ifndef NVBT_STAGE288
#define NVBT_STAGE288 1   // 288 B host-ring records staged per warp in shared memory and written per ticket block
#endif
constexpr unsigned kSkipTag = 0x80000000u;   // a committed ticket that carries no record (288 B host ring)


// Ring backpressure: ticket t may be written once t < tail + cap. has_room() is the
// cheap check against the device-side cache of the host's consumer index; reserve() then waits on the host
// index (PCIe reads, poll_room() in a warp-uniform loop) and gives up if the host never freed a slot within
// st.wait_ns (10 s; NVBT_PRODUCER_WAIT_MS at channel open) or another producer already gave up (the record is
// then dropped and counted, never hangs the GPU).
__device__ __forceinline__ bool has_room(const DevState& st, unsigned long long t) {
  return t < *(volatile const unsigned long long*)st.tail_cache + st.cap;
}
// One poll of the host index for ticket t (waiting since t0): 1 = room (tail cache refreshed), -1 = give up
// (st.wait_ns without progress, or another producer already gave up), 0 = keep waiting.
__device__ __forceinline__ int poll_room(const DevState& st, unsigned long long t, unsigned long long t0) {
  if (*(volatile const unsigned long long*)st.dropped != 0) return -1;
  const unsigned long long tl = *(volatile const unsigned long long*)st.tail;
  if (t < tl + st.cap) { atomicMax(st.tail_cache, tl); return 1; }
  return globaltimer() - t0 > st.wait_ns ? -1 : 0;
}

#ifndef NVBT_HOOKS_EXPERIMENT
#define NVBT_HOOKS_EXPERIMENT 0   // timing experiments only (wrong results): 1 no CTA flush, 2 no bin init, 3 both
#endif
template <uint32_t T, class Prog>
struct Hooks {
  static constexpr int NPC = Prog::N;
  static constexpr bool kOn = T != 0;
  static constexpr bool kCount = (T & (TOOL_COUNT | TOOL_BB)) != 0;
  static constexpr bool kBB = (T & TOOL_BB) != 0;
  static constexpr bool kLoopFree = Prog::REG_LO > Prog::REG_HI;   // no register-mode (loop) sites
  static constexpr int kMaxWarps = 8;  // workload CTAs have 256 threads
  static constexpr int kThreads = 32 * kMaxWarps;
  static constexpr int kScratchWord0 = (NPC * SITE_WORDS + 66 + 3) & ~3;  // 16-byte aligned
  // 288 B host-ring records (EM §5) are staged per warp (one ticket block of up to kBlock records) and written
  // to the ring together, so the link sees whole 128 B lines except at the block's two ends
  // (programs whose largest block would need more than 18 KB of staging keep a ticket per record)
  static constexpr unsigned kBlock = max_block<Prog>();
  static constexpr bool kStage = NVBT_STAGE288 && (T & TOOL_TRACE) != 0 && (T & TOOL_TRACE_DEV) == 0 &&
                                 stage_trace<Prog>::value && kBlock * 288u * kMaxWarps <= 18432u;
  static constexpr int kStageWord0 = kScratchWord0 + SCRATCH_WORDS * kMaxWarps;
  static_assert(!kStage || kBlock >= 2, "a staged block must hold a 176 B wide pair (2 x 192 B)");
  static constexpr int kSmemWords = kOn ? kStageWord0 + (kStage ? kMaxWarps * (int)kBlock * 72 : 0) : 1;
  static_assert(!((T & TOOL_COUNT) && (T & TOOL_BB)), "COUNT and BBCOUNT are exclusive");

  const DevState& st;
  unsigned* sb;
  unsigned tA[NPC], dT[NPC], wI[NPC], dW[NPC], mN[NPC], mS[NPC], mL[NPC];
  unsigned hS, hL;            // lane-distributed: lane l counts events with S (L) == l + 1
  unsigned pwT, pwW;          // this warp's executed thread / warp instructions (PER_WARP)
  unsigned iters = 0;         // loop instances since the last spill() (warp-uniform)
  unsigned seq;               // records emitted by this warp in this launch
  unsigned long long hslot;   // device ring: next slot this warp holds, `held` slots from there
  unsigned held;
  unsigned char* dptr = nullptr;   // device ring (TOOL_TRACE_DEV): this lane's address word of the next held slot
  unsigned nst = 0;           // 288 B host ring: records staged in the held block (from hslot on)
  unsigned stg = 0;           // 288 B host ring: this warp's staging area (shared address)
  unsigned npend = 0;         // uncommitted records of this warp (warp-uniform)
  unsigned pend_val = 0;      // lane k: tag value of the k-th uncommitted record
  unsigned* pend_tag = nullptr;
  unsigned lane, lane1, lanebit, lmlt, gwarp, scr, sbase;

  __device__ __forceinline__ Hooks(const DevState& s, unsigned* smem) : st(s), sb(smem) {
    zero_range<0, NPC - 1>();
    hS = hL = pwT = pwW = seq = 0;
    hslot = 0; held = 0;
    lane = lane_id();
    lane1 = lane + 1u;
    lanebit = 1u << lane;
    lmlt = lanemask_lt();
    const unsigned tid = threadIdx.x + threadIdx.y * blockDim.x;
    gwarp = (st.cta_lo + blockIdx.x + blockIdx.y * gridDim.x) * ((blockDim.x * blockDim.y) >> 5) + (tid >> 5);  // logical CTA
    scr = (unsigned)__cvta_generic_to_shared(sb + kScratchWord0 + SCRATCH_WORDS * ((tid >> 5) & (kMaxWarps - 1)));
    if constexpr (kStage) stg = (unsigned)__cvta_generic_to_shared(sb + kStageWord0 + 72 * (int)kBlock * ((tid >> 5) & (kMaxWarps - 1)));
    sbase = (unsigned)__cvta_generic_to_shared(sb);
    if constexpr (kOn && !(NVBT_HOOKS_EXPERIMENT & 2)) {
      // (CTAs of exactly kThreads threads; fixed-stride loops avoid a run-time trip-count division)
      constexpr int kInit = (T & TOOL_MEM) ? kSmemWords : kScratchWord0;   // scratch only for divergence
#pragma unroll
      for (int k = 0; k < (kInit + kThreads - 1) / kThreads; ++k) {
        const int i = (int)tid + k * kThreads;
        if (i < kInit) sb[i] = i < kScratchWord0 ? 0u : scratch_init_word((i - kScratchWord0) % SCRATCH_WORDS);
      }
      __syncthreads();
    }
  }

  // Active mask of the current basic-block instance: A = lanes with in_flow (EM §1). A is the same for
  // every pc of a basic block ("each thread will execute without change in control flow", P:L116 (§4)),
  // so kernels take one ballot per block instance and hand it to that block's hooks.
  struct Act { unsigned A; };
  // Debug builds (libnvbt_debug.so, -DNVBT_CHECK_CONVERGED) check the converged-hook discipline at every
  // hook: all 32 lanes of the warp must arrive together (R-15); a violation traps the kernel.
  __device__ __forceinline__ static void check_converged() {
#ifdef NVBT_CHECK_CONVERGED
    if (__activemask() != FULL) __trap();
#endif
  }
  __device__ __forceinline__ Act active(bool in_flow) const {
    check_converged();
    if constexpr (kOn) return Act{__ballot_sync(FULL, in_flow)};
    else return Act{0u};
  }

  // Injection point `PC` of the block whose active mask is `m`: pred = the lane's guard predicate
  // (only read for guarded pcs; false for lanes outside A), addr = effective address (memory pcs).
  template <int PC>
  __device__ __forceinline__ void at(Act m, bool pred = true, unsigned long long addr = 0) {
    constexpr nvbt_instr_desc d = Prog::t[PC];
    constexpr bool mem = is_mem_kind(d.kind);
    constexpr bool cnt = (T & TOOL_COUNT) || ((T & TOOL_BB) && (d.is_leader || d.guarded));
    constexpr bool div = mem && (T & TOOL_MEM);
    constexpr bool trc = mem && (T & TOOL_TRACE);
    constexpr bool reg = PC >= Prog::REG_LO && PC <= Prog::REG_HI;   // loop site: register counters
    check_converged();
    if constexpr (cnt || div || trc) {
      const unsigned A = m.A;
      const unsigned P = d.guarded ? (__ballot_sync(FULL, pred) & A) : A;
      const unsigned E = P;
      if constexpr (cnt) {
        const unsigned pa = __popc(A), wa = umin(pa, 1u);
        const unsigned pe = d.guarded ? __popc(E) : pa, we = d.guarded ? umin(pe, 1u) : wa;
        if constexpr (reg) {
          tA[PC] += pa;
          wI[PC] += wa;
          if constexpr (d.guarded) {
            dT[PC] += pa - pe;
            dW[PC] += wa - we;
          }
        } else {
          // one lane adds the hook's bins. Loop-free programs group the reductions under one branch
          // (ptxas does not predicate shared atomics: each separately predicated one costs its own
          // branch); programs with register-mode loops keep them separate (grouping raises the register
          // pressure of their loop bodies)
          const unsigned b = sbase + 4u * (PC * SITE_WORDS);
          if constexpr (kLoopFree) {
            if (lane == 0u) {
              red(b, pa);
              red(b + 8u, wa);
              if constexpr (d.guarded) {
                red(b + 4u, pa - pe);
                red(b + 12u, wa - we);
              }
            }
          } else {
            red_if(lane == 0u, b, pa);
            red_if(lane == 0u, b + 8u, wa);
            if constexpr (d.guarded) {
              red_if(lane == 0u, b + 4u, pa - pe);
              red_if(lane == 0u, b + 12u, wa - we);
            }
          }
          // this warp's executed totals (PER_WARP); register sites add theirs at retire()
          if constexpr ((T & TOOL_COUNT) != 0) {
            pwT += pe;
            pwW += we;
          } else {
            if constexpr (d.is_leader) {
              constexpr unsigned len = (unsigned)bb_len<Prog>(PC);
              pwT += len * pa;
              pwW += len * wa;
            }
            if constexpr (d.guarded) {
              pwT -= pa - pe;
              pwW -= wa - we;
            }
          }
        }
      }
      if constexpr (div || trc) {
        if (E != 0u) {
          if constexpr (div) {
            unsigned S, L;
            sectors_lines(addr, E, lane, lanebit, lmlt, scr, S, L);
            if constexpr (reg) {
              mN[PC] += 1u; mS[PC] += S; mL[PC] += L;
            } else {
              const unsigned b = sbase + 4u * (PC * SITE_WORDS);
              if constexpr (kLoopFree) {
                if (lane == 0u) {
                  red(b + 16u, 1u);
                  red(b + 20u, S);
                  red(b + 24u, L);
                }
              } else {
                red_if(lane == 0u, b + 16u, 1u);
                red_if(lane == 0u, b + 20u, S);
                red_if(lane == 0u, b + 24u, L);
              }
            }
            inc_if_eq(hS, S, lane1);
            inc_if_eq(hL, L, lane1);
          }
          if constexpr (trc) emit<PC>(A, P, (E & lanebit) != 0u, addr);
        }
      }
    }
  }

  __device__ __forceinline__ static void red(unsigned saddr, unsigned v) {
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
  }
  __device__ __forceinline__ static void red_if(bool p, unsigned saddr, unsigned v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.shared.add.u32 [%0], %1;\n\t}"
                 ::"r"(saddr), "r"(v), "r"((unsigned)p) : "memory");
  }

  // a6 producer. One record per executed global-memory event: lane 0 takes a ticket; the warp writes
  // the record with ONE 16 B-per-lane store (header with a zero tag + addresses) straight into the
  // pinned host ring. Commits are batched: lane (k % 32) remembers the tag word of the warp's k-th
  // uncommitted slot, and commit() makes every pending payload visible system-wide (one fence per lane
  // per batch instead of one per record) before the tags are stored. A warp commits before it can block
  // on a full ring, so reserved-but-uncommitted slots never stall the consumer for ever.
  // Compact channels (st.compact, EM §5.1, F3) send base + 32-bit deltas in one 176 B slot, or two slots
  // of 16 full addresses each when the warp's addresses span more than ±2 GB.
  // Device ring (F2): k contiguous slots from this SM's current chunk; the warp whose range covers the
  // chunk's end opens the stripe's next chunk. No backpressure: a ring without free chunks drops.
  // The whole warp runs the (rarely repeated) loop; lane 0 does the atomics and broadcasts, so no lane
  // is left behind in a divergent retry loop (the hooks that follow need the warp converged, R-15).
  __device__ __forceinline__ bool reserve_dev(unsigned k, unsigned long long& t) {
    const unsigned sm = smid();
    unsigned long long* w = st.rheads + (sm < st.rstripes ? sm : sm % st.rstripes);
    const unsigned long long t0 = globaltimer();
    bool ok = false;
    for (;;) {
      unsigned long long v = 0;
      if (lane == 0) v = atomicAdd(w, (unsigned long long)k);
      v = __shfl_sync(FULL, v, 0);
      const unsigned ck = (unsigned)(v >> 32), off = (unsigned)v;
      if (ck == kRingFull) break;
      if (off + k <= kRingChunk) {
        t = (unsigned long long)ck * kRingChunk + off;
        ok = t + k <= st.cap;
        break;
      }
      if (off <= kRingChunk) {   // this warp's range covers the chunk end: open the next chunk
        unsigned long long nc = 0;
        if (lane == 0) nc = atomicAdd(st.rheads + st.rstripes, 1ull);
        nc = __shfl_sync(FULL, nc, 0);
        if (nc * kRingChunk >= st.cap) {
          if (lane == 0) atomicExch(w, (unsigned long long)kRingFull << 32);
          break;
        }
        if (lane == 0) atomicExch(w, (nc << 32) | k);
        t = nc * kRingChunk;
        ok = t + k <= st.cap;
        break;
      }
      // another warp is opening the next chunk: wait until the stripe word moves on
      bool moved = false;
      while (!moved && globaltimer() - t0 < 2000000000ull) {
        unsigned c = 0;
        if (lane == 0) c = (unsigned)(*(volatile unsigned long long*)w >> 32);
        moved = __shfl_sync(FULL, c, 0) != ck;
      }
      if (!moved) break;
    }
    if (!ok && lane == 0) atomicAdd(st.dropped, 1ull);
    __syncwarp();
    return ok;
  }

  __device__ __forceinline__ bool reserve(unsigned k, unsigned long long& t) {
    int room = 1;
    if (lane == 0) {
      t = atomicAdd(st.head, (unsigned long long)k);
      room = has_room(st, t + k - 1);
    }
    t = __shfl_sync(FULL, t, 0);
    if (!__shfl_sync(FULL, room, 0)) {
      commit();
      // wait for the host to free the slot: the whole warp loops (lane 0 polls, then broadcasts), so
      // no lane stays behind in a divergent spin (R-15)
      int ok = 0;
      if (!st.no_wait) {
        const unsigned long long t0 = globaltimer();
        for (;;) {
          int r = 0;   // 1: room, -1: give up, 0: keep waiting
          if (lane == 0) r = poll_room(st, t + k - 1, t0);
          r = __shfl_sync(FULL, r, 0);
          if (r != 0) { ok = r > 0; break; }
          __nanosleep(500);
        }
      }
      if (!ok) {
        if (lane == 0) atomicAdd(st.dropped, 1ull);
        __syncwarp();
        return false;
      }
      __syncwarp();
    }
    return true;
  }

  // Slot of ticket t, its commit tag (lap + 1) and the tag's word in the dense tag array. The tags live
  // apart from the records: a 4 B tag store into a record's header line is a partial-line PCIe write of
  // its own per record, while tags of neighbouring tickets share lines of the tag array
  // (tools/peaks/d2h_protocol.cu: 39.7 -> 46.3 GB/s for the C4 emission pattern).
  __device__ __forceinline__ unsigned char* slot_ptr(unsigned long long t, unsigned& tag, unsigned*& tp) const {
    const unsigned long long lap = t / st.cap, i = t - lap * st.cap;
    tag = (unsigned)lap + 1u;
    tp = st.tags + i;
    return st.ring + i * st.slot_bytes;
  }

  __device__ __forceinline__ void add_pending(unsigned* tp, unsigned tag) {
    if (lane == npend) {
      pend_tag = tp;
      pend_val = tag;
    }
    if (++npend == 32) commit();
  }

  template <int PC>
  __device__ __forceinline__ void emit(unsigned A, unsigned P, bool act, unsigned long long addr) {
    constexpr nvbt_instr_desc d = Prog::t[PC];
    const unsigned w2 = (unsigned)d.opcode | ((unsigned)d.width << 16) | ((unsigned)d.kind << 24);
    const unsigned long long a = act ? addr : 0ull;
    if constexpr ((T & TOOL_TRACE_DEV) != 0) {
      // device ring, selected at compile time: a warp reserves the slots of the rest of its basic block
      // at once (x4 in loops) and walks them with a per-lane pointer (+288 B per record); every lane
      // stores its address (8 B, 256 B coalesced per record) and lanes 0, 1 the 32 B header with tag 1
      // in one predicated 16 B store each. Every slot is lap 1 and the consumer is a later kernel: no
      // fence, no commit.
      constexpr unsigned K = (unsigned)mem_left<Prog>(PC) * ((PC >= Prog::REG_LO && PC <= Prog::REG_HI) ? 4u : 1u);
      if (held == 0u) {   // warp-uniform
        unsigned long long t0;
        if (reserve_dev(K, t0)) {
          held = K;
          dptr = st.ring + t0 * RECORD_BYTES + 32u + 8u * lane;
        }
      }
      if (held != 0u) {
        --held;
        asm volatile("st.global.u64 [%0], %1;" ::"l"(dptr), "l"(a) : "memory");
        const bool l0 = lane == 0u;
        asm volatile("{\n\t.reg .pred p;\n\tsetp.lt.u32 p, %0, 2;\n\t@p st.global.v4.u32 [%1], {%2, %3, %4, %5};\n\t}"
                     ::"r"(lane), "l"(dptr + (8 * (int)lane - 32)), "r"(l0 ? st.launch : A), "r"(l0 ? gwarp : P),
                     "r"(l0 ? seq : w2), "r"(l0 ? (unsigned)PC : 1u) : "memory");
        __syncwarp();   // ptxas may branch around the predicated store: rejoin before the next hook (R-15)
        dptr += RECORD_BYTES;
      }
      ++seq;
      return;
    }
    unsigned long long t;
    unsigned tag;
    if (!st.compact) {
      bool have;
      if (st.no_wait) {
        // device ring: a warp reserves the slots of the rest of its basic block at once (x4 in loops)
        // and carries unused ones over; every slot is lap 1 and the consumer is a later kernel, so the
        // tag goes out with the header (no fence, no batched commit)
        constexpr unsigned K = (unsigned)mem_left<Prog>(PC) * ((PC >= Prog::REG_LO && PC <= Prog::REG_HI) ? 4u : 1u);
        have = held != 0u || reserve_dev(K, hslot);
        if (have) {
          held = held ? held : K;
          t = hslot++;
          --held;
        }
      } else {
        if constexpr (kStage) {   // host ring: stage into the warp's block, written when the block is full
          if (held == 0u) {       // warp-uniform; nothing staged
            constexpr unsigned K = block_at<Prog>(PC);
            const unsigned k = (unsigned)((unsigned long long)K < st.cap ? K : st.cap);
            if (reserve(k, hslot)) { held = k; nst = 0; }
          }
          if (held != 0u) {
            const unsigned src = 2u * (lane - 2u);
            const unsigned long long a0 = __shfl_sync(FULL, a, src & 31u), a1 = __shfl_sync(FULL, a, (src + 1u) & 31u);
            if (lane < 18) {
              const uint4 v = lane == 0   ? make_uint4(st.launch, gwarp, seq, (unsigned)PC)
                              : lane == 1 ? make_uint4(A, P, w2, 0u)
                                          : make_uint4((unsigned)a0, (unsigned)(a0 >> 32), (unsigned)a1, (unsigned)(a1 >> 32));
              asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(stg + 288u * nst + 16u * lane),
                           "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
            }
            ++nst;
            --held;
            if (held == 0u) flush288();
          }
          ++seq;
          return;
        }
        have = reserve(1, t);
      }
      if (have) {
        if (st.no_wait) {
          // device ring (HBM, issue-bound producer): every lane stores its own address (8 B, 256 B
          // coalesced per record) and lanes 0, 1 the 32 B header with tag 1 — no shuffles
          unsigned char* rec = st.ring + t * RECORD_BYTES;
          *reinterpret_cast<unsigned long long*>(rec + 32 + 8 * lane) = a;
          if (lane < 2) {
            const uint4 v = lane == 0 ? make_uint4(st.launch, gwarp, seq, (unsigned)PC) : make_uint4(A, P, w2, 1u);
            *reinterpret_cast<uint4*>(rec + 16 * lane) = v;
          }
        } else {
          unsigned* tp;
          unsigned char* rec = slot_ptr(t, tag, tp);
          // pinned host ring: one 16 B-per-lane store per record. Lane j < 18 writes bytes
          // [16j, 16j + 16): lanes 0, 1 the header (tag 0), lane j >= 2 the addresses of lanes 2(j-2),
          // 2(j-2)+1
          const unsigned src = 2u * (lane - 2u);
          const unsigned long long a0 = __shfl_sync(FULL, a, src & 31u), a1 = __shfl_sync(FULL, a, (src + 1u) & 31u);
          if (lane < 18) {
            const uint4 v = lane == 0   ? make_uint4(st.launch, gwarp, seq, (unsigned)PC)
                            : lane == 1 ? make_uint4(A, P, w2, 0u)
                                        : make_uint4((unsigned)a0, (unsigned)(a0 >> 32), (unsigned)a1, (unsigned)(a1 >> 32));
            *reinterpret_cast<uint4*>(rec + 16 * lane) = v;
          }
          add_pending(tp, tag);
        }
      }
      ++seq;
      return;
    }
    const unsigned E = P;
    const unsigned long long base = __shfl_sync(FULL, addr, __ffs(E) - 1);
    const long long dl = (long long)(addr - base);
    if (st.compact >= 3u) {
      // 128 B slots (EM §5.2): one whole PCIe line per record when every lane of E is within +-32 KB of
      // the first (header, base, 32 x i16 deltas), else three slots of full addresses. Slots come from a
      // block of consecutive tickets the warp reserves for the rest of its basic block (x4 in loops), so
      // the warp's records and commit tags are contiguous on the link (tools/peaks/d2h_line.cu: 309 ->
      // 387 M lines/s); slots the block does not use are committed as skip slots (EM §5.2, flags 0xC0).
      constexpr unsigned K = (unsigned)mem_left<Prog>(PC) * ((PC >= Prog::REG_LO && PC <= Prog::REG_HI) ? 4u : 1u);
      const bool shortf = st.compact == 3u && __all_sync(FULL, !act || (dl >= -32768ll && dl <= 32767ll));
      const unsigned need = shortf ? 1u : 3u;
      bool have = true;
      if (held < need) {                           // warp-uniform
        release();
        const unsigned long long want = (unsigned long long)(K > need ? K : need);
        const unsigned k = (unsigned)(want < st.cap ? want : st.cap);   // a block never exceeds the ring
        have = reserve(k, hslot);
        held = have ? k : 0u;
        nst = 0;
      }
      // staged (kStage): the block's lines are formed in shared memory and written together (flush_line)
      unsigned lidx = 0;
      if (have) {
        if constexpr (kStage) {
          lidx = nst;
          nst += need;
        } else {
          t = hslot;
          hslot += need;
        }
        held -= need;
      }
      if (have && shortf) {
        {
          unsigned* tp = nullptr;
          unsigned char* rec = nullptr;
          if constexpr (!kStage) rec = slot_ptr(t, tag, tp);
          // u32 word k of the delta area (bytes 40..103) = delta[2k] | delta[2k + 1] << 16, built on lane 2k
          const unsigned d16 = act ? ((unsigned)dl & 0xFFFFu) : 0u;
          const unsigned wp = d16 | (__shfl_down_sync(FULL, d16, 1) << 16);
          // chunk c = bytes 16c .. 16c + 15: 0, 1 header; 2 base + words 0, 1; 3..5 words 4c - 10 ..; 6 words
          // 14, 15; 7 zero
          const int k0 = lane == 2u ? 0 : lane == 6u ? 14 : 4 * (int)lane - 10;
          const unsigned s0 = (2u * (unsigned)k0) & 31u;
          const unsigned u0 = __shfl_sync(FULL, wp, s0), u1 = __shfl_sync(FULL, wp, (s0 + 2u) & 31u);
          const unsigned u2 = __shfl_sync(FULL, wp, (s0 + 4u) & 31u), u3 = __shfl_sync(FULL, wp, (s0 + 6u) & 31u);
          if (lane < 8) {
            const uint4 v = lane == 0   ? make_uint4(st.launch, gwarp, seq, (unsigned)PC)
                            : lane == 1 ? make_uint4(A, P, w2 | 0x80000000u, 0u)
                            : lane == 2 ? make_uint4((unsigned)base, (unsigned)(base >> 32), u0, u1)
                            : lane <= 5 ? make_uint4(u0, u1, u2, u3)
                            : lane == 6 ? make_uint4(u0, u1, 0u, 0u)
                                        : make_uint4(0u, 0u, 0u, 0u);
            if constexpr (kStage) sts_v4(stg + 128u * lidx + 16u * lane, v);
            else *reinterpret_cast<uint4*>(rec + 16 * lane) = v;
          }
          if constexpr (!kStage) add_pending(tp, tag);
        }
      } else if (have) {
        // three slots: slot 0 = header (kind | 0x40) + lanes 0..11; slots 1, 2 carry flag 0x20 at byte 27
        // and lanes 12..26 (bytes 0..23: 3 lanes, 32..127: 12 lanes) and 27..31
        unsigned tg[3] = {0u, 0u, 0u};
        unsigned* tps[3] = {nullptr, nullptr, nullptr};
        unsigned char* r[3] = {nullptr, nullptr, nullptr};
        if constexpr (!kStage) {
#pragma unroll
          for (int k = 0; k < 3; ++k) r[k] = slot_ptr(t + k, tg[k], tps[k]);
        }
        const unsigned sl = lane >> 3, c = lane & 7u;
        // first lane of the chunk's address pair: slot 0 chunk c >= 2: 2(c-2); slots 1, 2: chunk 0 -> 12 + 15(s-1),
        // chunk 1 -> 14 + 15(s-1) (one address + the flag word), chunk c >= 2 -> 15 + 15(s-1) + 2(c-2)
        const unsigned src = sl == 0u ? 2u * (c - 2u) : (15u * (sl - 1u) + (c == 0u ? 12u : c == 1u ? 14u : 15u + 2u * (c - 2u)));
        const unsigned long long a0 = __shfl_sync(FULL, a, src & 31u), a1 = __shfl_sync(FULL, a, (src + 1u) & 31u);
        if (lane < 24) {
          const bool hdr = sl == 0u && c < 2u;
          const bool flagw = sl != 0u && c == 1u;
          const bool zero = sl == 2u && c >= 3u;
          const uint4 v = hdr ? (c == 0u ? make_uint4(st.launch, gwarp, seq, (unsigned)PC) : make_uint4(A, P, w2 | 0x40000000u, 0u))
                        : flagw ? make_uint4((unsigned)a0, (unsigned)(a0 >> 32), 0x20000000u, 0u)
                        : zero ? make_uint4(0u, 0u, 0u, 0u)
                               : make_uint4((unsigned)a0, (unsigned)(a0 >> 32), (unsigned)a1, (unsigned)(a1 >> 32));
          if constexpr (kStage) sts_v4(stg + 128u * (lidx + sl) + 16u * c, v);
          else *reinterpret_cast<uint4*>(r[sl] + 16 * c) = v;
        }
        if constexpr (!kStage) {
          add_pending(tps[0], tg[0]);
          add_pending(tps[1], tg[1]);
          add_pending(tps[2], tg[2]);
        }
      }
      if constexpr (kStage) {
        if (have && held == 0u) flush_line();
      }
      ++seq;
      return;
    }
    // 176 B slots: tickets from the warp's block as for 128 B slots (skip slots for the unused ones)
    const bool shortc = st.compact == 1u && __all_sync(FULL, !act || (dl >= -0x80000000ll && dl <= 0x7fffffffll));
    const unsigned needc = shortc ? 1u : 2u;
    bool havec = true;
    if (held < needc) {                            // warp-uniform
      release();
      constexpr unsigned K = (unsigned)mem_left<Prog>(PC) * ((PC >= Prog::REG_LO && PC <= Prog::REG_HI) ? 4u : 1u);
      const unsigned long long want = (unsigned long long)(K > needc ? K : needc);
      const unsigned k = (unsigned)(want < st.cap ? want : st.cap);
      havec = reserve(k, hslot);
      held = havec ? k : 0u;
      nst = 0;
    }
    // staged (kStage): slots are formed in the warp's shared-memory block and written with the block
    // (flush_c176), 192 B apart as in the ring; else straight into the ring
    unsigned idx = 0;
    if (havec) {
      if constexpr (kStage) {
        idx = nst;
        nst += needc;
      } else {
        t = hslot;
        hslot += needc;
      }
      held -= needc;
    }
    if (havec && shortc) {
      {
        unsigned* tp = nullptr;
        unsigned char* rec = nullptr;
        if constexpr (!kStage) rec = slot_ptr(t, tag, tp);
        // 11 chunks: header, header (kind | 0x80), base, then 4 deltas per chunk (lanes 4(j-3) .. +3)
        const unsigned dd = act ? (unsigned)dl : 0u;
        const unsigned s0 = 4u * (lane - 3u);
        const unsigned d0 = __shfl_sync(FULL, dd, s0 & 31u), d1 = __shfl_sync(FULL, dd, (s0 + 1u) & 31u);
        const unsigned d2 = __shfl_sync(FULL, dd, (s0 + 2u) & 31u), d3 = __shfl_sync(FULL, dd, (s0 + 3u) & 31u);
        if (lane < 11) {
          const uint4 v = lane == 0   ? make_uint4(st.launch, gwarp, seq, (unsigned)PC)
                          : lane == 1 ? make_uint4(A, P, w2 | 0x80000000u, 0u)
                          : lane == 2 ? make_uint4((unsigned)base, (unsigned)(base >> 32), 0u, 0u)
                                      : make_uint4(d0, d1, d2, d3);
          if constexpr (kStage) sts_v4(stg + 192u * idx + 16u * lane, v);
          else *reinterpret_cast<uint4*>(rec + 16 * lane) = v;
        }
        if constexpr (!kStage) add_pending(tp, tag);
      }
    } else if (havec) {
      // wide pair: slot t = lanes 0-15, slot t+1 = lanes 16-31 (full addresses); lanes 0-9 write the
      // first slot's 10 chunks, lanes 16-25 the second's
      unsigned tag0 = 0, tag1 = 0;
      unsigned *tp0 = nullptr, *tp1 = nullptr;
      unsigned char *r0 = nullptr, *r1 = nullptr;
      if constexpr (!kStage) {
        r0 = slot_ptr(t, tag0, tp0);
        r1 = slot_ptr(t + 1, tag1, tp1);
      }
      const unsigned h = lane >> 4, j = lane & 15u;
      const unsigned src = 16u * h + 2u * (j - 2u);
      const unsigned long long a0 = __shfl_sync(FULL, a, src & 31u), a1 = __shfl_sync(FULL, a, (src + 1u) & 31u);
      if (j < 10) {
        const unsigned flag = h ? 0x20000000u : 0x40000000u;
        const uint4 v = j == 0   ? make_uint4(st.launch, gwarp, seq, (unsigned)PC)
                        : j == 1 ? make_uint4(A, P, w2 | flag, 0u)
                                 : make_uint4((unsigned)a0, (unsigned)(a0 >> 32), (unsigned)a1, (unsigned)(a1 >> 32));
        if constexpr (kStage) sts_v4(stg + 192u * (idx + h) + 16u * j, v);
        else *reinterpret_cast<uint4*>((h ? r1 : r0) + 16 * j) = v;
      }
      if constexpr (!kStage) {
        add_pending(tp0, tag0);
        add_pending(tp1, tag1);
      }
    }
    if constexpr (kStage) {
      if (havec && held == 0u) flush_c176();
    }
    ++seq;
  }

  __device__ __forceinline__ void sts_v4(unsigned a, const uint4& v) {
    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
  }

  // Staged ticket blocks (kStage): writes the warp's n_data staged slots (stride bytes apart in shared memory
  // and in the ring; Q 16 B chunks each) to ring tickets hslot .. hslot + n_data - 1, 16 B per lane per step
  // over the whole run (contiguous except where the ring wraps), then commits tickets hslot .. + n_tags - 1:
  // those past n_data with the skip bit (no record).
  template <unsigned Q>
  __device__ __forceinline__ void write_block(unsigned n_data, unsigned n_tags, unsigned stride) {
    __syncwarp();
    for (unsigned c = lane; c < Q * n_data; c += 32u) {
      const unsigned r = c / Q, q = c - Q * r;
      unsigned tg;
      unsigned* tp;
      unsigned char* rec = slot_ptr(hslot + r, tg, tp);
      uint4 v;
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                   : "r"(stg + stride * r + 16u * q) : "memory");
      *reinterpret_cast<uint4*>(rec + 16u * q) = v;
    }
    for (unsigned r = 0; r < n_tags; ++r) {       // warp-uniform
      unsigned tg;
      unsigned* tp;
      slot_ptr(hslot + r, tg, tp);
      add_pending(tp, r < n_data ? tg : (tg | kSkipTag));
    }
    hslot += n_tags;
    held = 0;
    nst = 0;
    __syncwarp();                                 // staging reads done before the next block's stores
  }

  // 176 B slots: the block's unused slots become skip slots in shared memory (0xC0 at byte 27), and all of
  // them go out with the block (192 B apart, the pad included; two slots = three whole lines).
  __device__ __forceinline__ void flush_c176() {
    if constexpr (kStage) {
      if (lane < held) sts_v4(stg + 192u * (nst + lane) + 16u, make_uint4(0u, 0u, 0xC0000000u, 0u));
      const unsigned n = nst + held;
      write_block<12>(n, n, 192u);
    }
  }

  // 128 B line slots: as for 176 B slots, 128 B apart (each slot one whole line)
  __device__ __forceinline__ void flush_line() {
    if constexpr (kStage) {
      if (lane < held) sts_v4(stg + 128u * (nst + lane) + 16u, make_uint4(0u, 0u, 0xC0000000u, 0u));
      const unsigned n = nst + held;
      write_block<8>(n, n, 128u);
    }
  }

  // 288 B records: the staged records go out with the block; its unused tickets are committed with the skip
  // bit in their tags, no data.
  __device__ __forceinline__ void flush288() {
    if constexpr (kStage) write_block<18>(nst, nst + held, 288u);
  }

  // Compact transports: the rest of the warp's ticket block goes out now, its unused tickets as skip slots
  // (header chunk with flags 0xC0 at byte 27, committed like records) so the consumer can pass them.
  // Kernels without staging write the skip headers straight into the ring.
  __device__ __forceinline__ void release() {
    if constexpr (kStage) {
      if (held != 0u || nst != 0u) {
        if (st.compact <= 2u) flush_c176();        // 176 B slots, staged
        else flush_line();                         // 128 B line slots, staged
      }
    } else {
      release_unstaged();
    }
  }
  __device__ __forceinline__ void release_unstaged() {
    while (held != 0u) {                           // warp-uniform
      const unsigned k = held < 32u ? held : 32u;
      unsigned tag = 0;
      unsigned* tp = nullptr;
      unsigned char* rec = slot_ptr(hslot + (lane < k ? lane : 0u), tag, tp);
      if (lane < k) *reinterpret_cast<uint4*>(rec + 16) = make_uint4(0u, 0u, 0xC0000000u, 0u);
      for (unsigned i = 0; i < k; ++i) {
        const unsigned ti = __shfl_sync(FULL, tag, i);
        unsigned* tpi = reinterpret_cast<unsigned*>(__shfl_sync(FULL, reinterpret_cast<unsigned long long>(tp), i));
        add_pending(tpi, ti);
      }
      hslot += k;
      held -= k;
    }
  }

  __device__ __forceinline__ void commit() {
    if (npend == 0) return;
    __threadfence_system();   // this lane's payload stores are performed system-wide ...
    __syncwarp();             // ... for every lane, before any tag below is written
    if (lane < npend)
      asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(pend_tag), "r"(pend_val) : "memory");
    npend = 0;
  }

  // executed-instruction totals of pc range [LO, HI] (for PER_WARP), BB-derived where needed
  template <int PC>
  __device__ __forceinline__ void texe(unsigned& t, unsigned& w) const {
    constexpr nvbt_instr_desc d = Prog::t[PC];
    if constexpr ((T & TOOL_COUNT) || d.is_leader || d.guarded) {
      t += tA[PC] - dT[PC];
      w += wI[PC] - dW[PC];
    } else if constexpr (kBB) {
      constexpr int L = leader_of<Prog>(PC);
      t += tA[L];
      w += wI[L];
    }
  }

  // Moves the register counters of pcs [LO, HI] into the CTA's shared bins (lane-parallel: lane l takes
  // pc LO + 32r + l) and zeroes them, freeing their registers. In BB mode [LO, HI] must be whole blocks.
  template <int LO, int HI>
  __device__ __forceinline__ void retire() {
    constexpr int RLO = LO > Prog::REG_LO ? LO : Prog::REG_LO;
    constexpr int RHI = HI < Prog::REG_HI ? HI : Prog::REG_HI;
    if constexpr (kOn && RLO <= RHI) retire_regs<RLO, RHI>();
  }

  // register-mode pcs [LO, HI] -> shared bins
  template <int LO, int HI>
  __device__ __forceinline__ void retire_regs() {
    if constexpr (kOn) {
      static_assert(LO >= 0 && HI < NPC && LO <= HI, "bad range");
      static_assert(!kBB || (Prog::t[LO].is_leader && (HI + 1 == NPC || Prog::t[HI + 1].is_leader)),
                    "register-mode pc ranges are whole basic blocks");
      if constexpr (kCount) {
        unsigned t = 0, w = 0;
        retire_sum<LO, HI>(t, w);
        pwT += t; pwW += w;
      }
      retire_round<LO, HI, LO>();
      zero_range<LO, HI>();
    }
  }

  template <int LO, int HI, int BASE>
  __device__ __forceinline__ void retire_round() {
    if constexpr (BASE <= HI) {
      unsigned v[SITE_WORDS] = {0, 0, 0, 0, 0, 0, 0};
      select_lane<BASE, (HI < BASE + 31 ? HI : BASE + 31), BASE>(v);
      if (BASE + (int)lane <= HI) {
        const int pc = BASE + (int)lane;
#pragma unroll
        for (int k = 0; k < SITE_WORDS; ++k)
          if (v[k]) atomicAdd(&sb[pc * SITE_WORDS + k], v[k]);
      }
      retire_round<LO, HI, BASE + 32>();
    }
  }

  template <int PC, int END, int BASE>
  __device__ __forceinline__ void select_lane(unsigned (&v)[SITE_WORDS]) const {
    if constexpr (PC <= END) {
      const bool me = lane == (unsigned)(PC - BASE);
      v[0] = me ? tA[PC] : v[0]; v[1] = me ? dT[PC] : v[1]; v[2] = me ? wI[PC] : v[2]; v[3] = me ? dW[PC] : v[3];
      v[4] = me ? mN[PC] : v[4]; v[5] = me ? mS[PC] : v[5]; v[6] = me ? mL[PC] : v[6];
      select_lane<PC + 1, END, BASE>(v);
    }
  }

  template <int LO, int HI>
  __device__ __forceinline__ void zero_range() {
    if constexpr (LO <= HI) {
      tA[LO] = dT[LO] = wI[LO] = dW[LO] = mN[LO] = mS[LO] = mL[LO] = 0;
      zero_range<LO + 1, HI>();
    }
  }

  template <int LO, int HI>
  __device__ __forceinline__ void retire_sum(unsigned& t, unsigned& w) const {
    if constexpr (LO <= HI) {
      texe<LO>(t, w);
      retire_sum<LO + 1, HI>(t, w);
    }
  }

  // Overflow guard for loops. Every register / lane counter grows by at most 32 per loop instance and
  // per pc, and the CTA's shared bins hold 8 warps' worth, so all stay below 2^28 as long as no warp
  // keeps more than 2^20 instances in them: kernels run their loops in chunks of kSpillEvery instances
  // and call spill() between chunks (or tick() once per instance), which moves this warp's register-mode
  // counters, divergence histogram lanes and per-warp totals straight into the global 64-bit bins
  // (lane-parallel atomics) and zeroes them. Without it an SGEMM with K >= 2^24 (or a BFS hub of that
  // degree) would wrap a u32 bin silently.
  static constexpr unsigned kSpillEvery = 1u << 20;
  __device__ __forceinline__ void tick() {
    if constexpr (kOn && !kLoopFree) {
      if (++iters == kSpillEvery) {
        iters = 0;
        spill();
      }
    }
  }
  __device__ __forceinline__ unsigned long long stripe_off() const {
    return (unsigned long long)((st.cta_lo + blockIdx.x + blockIdx.y * gridDim.x) & (st.stripes - 1u)) * st.stripe_words;
  }
  __device__ __forceinline__ void spill() {
    if constexpr (kOn && !kLoopFree) {
      constexpr int LO = Prog::REG_LO, HI = Prog::REG_HI;
      const unsigned long long so = stripe_off();
      if constexpr (kCount) {
        unsigned t = 0, w = 0;
        retire_sum<LO, HI>(t, w);
        pwT += t; pwW += w;
        if (st.pw != nullptr && lane == 0 && gwarp < st.n_warps) {
          if (pwT) atomicAdd(st.pw + gwarp, (unsigned long long)pwT);
          if (pwW) atomicAdd(st.pw + st.n_warps + gwarp, (unsigned long long)pwW);
        }
        pwT = pwW = 0;
      }
      spill_round<LO, HI, LO>(so);
      zero_range<LO, HI>();
      if (hS) atomicAdd(st.hist + so + 1 + lane, (unsigned long long)hS);
      if (hL) atomicAdd(st.hist + so + 34 + lane, (unsigned long long)hL);
      hS = hL = 0;
      __syncwarp();
    }
  }
  template <int LO, int HI, int BASE>
  __device__ __forceinline__ void spill_round(unsigned long long so) {
    if constexpr (BASE <= HI) {
      unsigned v[SITE_WORDS] = {0, 0, 0, 0, 0, 0, 0};
      select_lane<BASE, (HI < BASE + 31 ? HI : BASE + 31), BASE>(v);
      if (BASE + (int)lane <= HI) {
        const int pc = BASE + (int)lane;
        unsigned long long* s = st.site + so + 4 * pc;
        if (v[0]) atomicAdd(s + 0, (unsigned long long)v[0]);
        if (v[0] - v[1]) atomicAdd(s + 1, (unsigned long long)(v[0] - v[1]));
        if (v[2]) atomicAdd(s + 2, (unsigned long long)v[2]);
        if (v[2] - v[3]) atomicAdd(s + 3, (unsigned long long)(v[2] - v[3]));
        if (v[4]) {
          unsigned long long* m = st.mem + so + 3 * pc;
          atomicAdd(m + 0, (unsigned long long)v[4]);
          atomicAdd(m + 1, (unsigned long long)v[5]);
          atomicAdd(m + 2, (unsigned long long)v[6]);
        }
      }
      spill_round<LO, HI, BASE + 32>(so);
    }
  }

  // CTA epilogue (nvbt_cta_flush): registers -> shared bins -> one global atomic per non-zero bin.
  // Must be reached by every thread of the CTA.
  __device__ __forceinline__ void finish() {
    if constexpr (kOn) {
      if constexpr ((T & TOOL_TRACE) != 0 && (T & TOOL_TRACE_DEV) == 0) {
        if (st.compact != 0u) release();   // compact host rings take tickets in blocks
        else if (!st.no_wait && (held != 0u || nst != 0u)) flush288();
        commit();
      } else if constexpr ((T & TOOL_TRACE) != 0) {
        commit();
      }
      retire<0, NPC - 1>();
      if (hS) atomicAdd(&sb[NPC * SITE_WORDS + 1 + lane], hS);
      if (hL) atomicAdd(&sb[NPC * SITE_WORDS + 34 + lane], hL);
      if constexpr (kCount) {
        if (st.pw != nullptr && lane == 0 && gwarp < st.n_warps) {
          atomicAdd(st.pw + gwarp, (unsigned long long)pwT);
          atomicAdd(st.pw + st.n_warps + gwarp, (unsigned long long)pwW);
        }
      }
      if (NVBT_HOOKS_EXPERIMENT & 1) return;
      __syncthreads();
      const int tid = threadIdx.x + threadIdx.y * blockDim.x;
      constexpr int nt = kThreads;
      // this CTA's stripe of the global bins (spreads same-address atomics over st.stripes copies)
      // (logical CTA id: a partitioned launch fills the same stripes as the unpartitioned one)
      const unsigned long long so = stripe_off();
      for (int pc = tid; pc < NPC; pc += nt) {
        const unsigned* b = sb + pc * SITE_WORDS;
        if (b[0] | b[2]) {
          unsigned long long* s = st.site + so + 4 * pc;
          atomicAdd(s + 0, (unsigned long long)b[0]);
          if (b[0] - b[1]) atomicAdd(s + 1, (unsigned long long)(b[0] - b[1]));
          atomicAdd(s + 2, (unsigned long long)b[2]);
          if (b[2] - b[3]) atomicAdd(s + 3, (unsigned long long)(b[2] - b[3]));
        }
        if (b[4]) {
          unsigned long long* m = st.mem + so + 3 * pc;
          atomicAdd(m + 0, (unsigned long long)b[4]);
          atomicAdd(m + 1, (unsigned long long)b[5]);
          atomicAdd(m + 2, (unsigned long long)b[6]);
        }
      }
      for (int i = tid; i < 66; i += nt)
        if (sb[NPC * SITE_WORDS + i]) atomicAdd(st.hist + so + i, (unsigned long long)sb[NPC * SITE_WORDS + i]);
    }
  }
};

}  // namespace nvbt
