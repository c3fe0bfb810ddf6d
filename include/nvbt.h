/* nvbt — B200-native device-side instrumentation hot path of NVBit (Villa et al., MICRO'19).
 *
 * C ABI of libnvbt.so. Citations "P:Lnnn (§x)" are lines of /root/reference/PAPER.md; the event model
 * every call follows is docs/EVENT_MODEL.md (EM §n).
 *
 * Conventions (all entry points):
 *  - Every function returns int: NVBT_OK (0) or a negative nvbt_status. No C++ exception crosses the
 *    ABI. nvbt_last_error() returns a thread-local message for the last failing call on this thread.
 *  - Ownership: ALL device memory and pinned host memory are caller-owned (allocated by PyTorch). The
 *    library never calls cudaMalloc/cudaHostAlloc. Streams are caller-owned (cudaStream_t as void*).
 *  - Results are cumulative since nvbt_init / nvbt_reset, like NVBit's __managed__ counters read at
 *    nvbit_at_term (P:L190-192, P:L254-258 (§6.1)). Read calls synchronise the context's stream, run the
 *    fold kernel on it and copy into caller host buffers.
 *  - Device pointers passed to workload/replay calls must be 16-byte aligned device addresses.
 */
#ifndef NVBT_H
#define NVBT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NVBT_ABI_VERSION 1

enum nvbt_status {
  NVBT_OK = 0,
  NVBT_EINVAL = -1,     /* null pointer, size or flag mismatch */
  NVBT_ESTATE = -2,     /* feature not enabled at init, or channel not open */
  NVBT_ENOMEM = -3,     /* workspace or ring too small */
  NVBT_ECUDA = -4,      /* CUDA runtime error; message carries cudaGetErrorString */
  NVBT_ETIMEDOUT = -5,  /* channel drain timeout, or a producer gave up on backpressure */
  NVBT_EVERSION = -6    /* ABI version mismatch */
};

/* Context flags: what the context collects (EM §2). */
enum nvbt_flags {
  NVBT_COUNT = 1,       /* thread/warp issued/executed counts (Listing 1 tool, P:L80-89 (§3)) */
  NVBT_OPHIST = 2,      /* per-opcode histogram (§6.2 Top-5 tool) */
  NVBT_BB = 4,          /* per-basic-block entries/instructions (BB rule P:L115-117 (§4)) */
  NVBT_MEMDIV = 8,      /* unique 32B sectors / 128B lines per warp global LD/ST (Listing 8) */
  NVBT_PER_WARP = 16,   /* per-warp thread/warp executed counts (n_warps entries) */
  NVBT_TRACE = 32       /* per-warp address records through the device->host channel */
};

/* Per-launch tool selection for instrumented workload launches (the compiled-in analogue of
 * nvbit_insert_call + nvbit_enable_instrumented, P:L123, P:L169 (§4, §5.1)). */
enum nvbt_tools {
  NVBT_TOOL_NONE = 0,     /* uninstrumented launch of the same source (slowdown baseline) */
  NVBT_TOOL_COUNT = 1,    /* a hook at every pc: counts, opcode and BB histograms */
  NVBT_TOOL_BBCOUNT = 2,  /* hooks only at BB leaders and guarded pcs; per-pc counts derived */
  NVBT_TOOL_MEMDIV = 4,   /* hooks at global-memory pcs: sector/line divergence */
  NVBT_TOOL_TRACE = 8,    /* hooks at global-memory pcs: one 288 B record per executed event (EM §5) */
  NVBT_TOOL_EMU = 16      /* replace proxy instructions by their emulation function (F4, §6.3 P:L286-295;
                             only the WFFT32 proxy kernel has one, EM §3.6) */
};

enum nvbt_kind { NVBT_K_ALU = 0, NVBT_K_CTRL = 1, NVBT_K_GLD = 2, NVBT_K_GST = 3, NVBT_K_GATOM = 4,
                 NVBT_K_OTHERMEM = 5 };

/* One row of a program table ("virtual SASS", EM §3) — stands in for NVBit's class Instr. */
typedef struct {
  uint16_t opcode;
  uint8_t kind;       /* enum nvbt_kind */
  uint8_t width;      /* bytes per lane for memory kinds (1,2,4,8,16), else 0 */
  uint32_t bb;        /* basic block id */
  uint8_t is_leader;  /* first pc of its basic block */
  uint8_t guarded;    /* carries a guard predicate (P may differ from A) */
  uint16_t pad;
} nvbt_instr_desc;

typedef struct {
  uint32_t version;        /* NVBT_ABI_VERSION */
  int32_t device;          /* CUDA device ordinal the workspace lives on */
  void* stream;            /* cudaStream_t every call of this context is ordered on */
  const nvbt_instr_desc* prog;  /* host array [n_pcs], copied at init */
  uint32_t n_pcs;          /* 1..4096 */
  uint32_t n_opcodes;      /* 1..256, > every opcode in prog */
  uint32_t n_bbs;          /* > every bb in prog, <= n_pcs */
  uint32_t n_warps;        /* global warp ids are < n_warps when NVBT_PER_WARP (else ignored) */
  uint32_t flags;          /* enum nvbt_flags */
  void* d_workspace;       /* device memory, >= nvbt_workspace_size bytes, 256-byte aligned */
  size_t workspace_bytes;
} nvbt_config;

typedef struct nvbt_ctx_s* nvbt_ctx;
typedef struct nvbt_chan_s* nvbt_channel;

int nvbt_abi_version(void);
const char* nvbt_last_error(void);

/* Bytes of device workspace a config needs (only n_pcs, n_opcodes, n_bbs, n_warps, flags are read). */
int nvbt_workspace_size(const nvbt_config* cfg, size_t* bytes);

/* Validates cfg, uploads the program table into the workspace and zeroes the accumulators (on
 * cfg->stream). EINVAL on a malformed table or config, ENOMEM if the workspace is too small. */
int nvbt_init(const nvbt_config* cfg, nvbt_ctx* out);
int nvbt_reset(nvbt_ctx ctx);            /* zero accumulators and the launch counter (async on stream) */
int nvbt_fini(nvbt_ctx ctx);             /* frees host-side state only; closes an open channel */

/* The packed int64 accumulator region (device pointer + length in int64 words): per-pc site bins,
 * BB-mode bins, memory-divergence bins, S/L histograms and per-warp arrays. Sums of disjoint event
 * sets add elementwise, so a multi-GPU merge is one int64 SUM all-reduce of this region (EM §4). */
int nvbt_accum_view(nvbt_ctx ctx, void** d_ptr, size_t* n_int64);

/* accum += factor * src over the whole accumulator region (n_int64 words of nvbt_accum_view); src is a
 * device copy of another context's region with the same layout. Used by kernel sampling (F1,
 * P:L274-282 (§6.2)): the counts of the one instrumented launch of a grid shape are extrapolated to all
 * launches of that shape. Asynchronous on the context's stream. */
int nvbt_accum_axpy(nvbt_ctx ctx, const void* d_src, size_t n_int64, int64_t factor);

/* ---- read calls (EM §2); all synchronise the stream ---- */
typedef struct { uint64_t thread_issued, thread_exec, warp_issued, warp_exec; } nvbt_counts;
/* per_warp_thread / per_warp_warp: nullable host arrays [n_warps] (need NVBT_PER_WARP). */
int nvbt_count(nvbt_ctx ctx, nvbt_counts* out, uint64_t* per_warp_thread, uint64_t* per_warp_warp);
/* thread_exec / warp_exec: host arrays [n_opcodes]. */
int nvbt_opcode_hist(nvbt_ctx ctx, uint64_t* thread_exec, uint64_t* warp_exec, uint32_t n_opcodes);
typedef struct { uint64_t entries_warp, entries_thread, instrs_warp, instrs_thread; } nvbt_bb_stats;
int nvbt_bb_count(nvbt_ctx ctx, nvbt_bb_stats* out, uint32_t n_bbs);
typedef struct { uint64_t accesses, sectors, lines; } nvbt_memdiv;       /* per pc: n, ΣS, ΣL */
typedef struct { nvbt_memdiv sum; uint64_t hist_sectors[33], hist_lines[33]; } nvbt_memdiv_total;
/* per_pc: nullable host array [n_pcs]. The paper's printed figure is sum.lines/sum.accesses. */
int nvbt_mem_divergence(nvbt_ctx ctx, nvbt_memdiv* per_pc, uint32_t n_pcs, nvbt_memdiv_total* tot);

/* ---- trace channel (a6; "sent to the CPU for further processing", P:L187 (§6.1)) ----
 * pinned_ring: caller-owned pinned, device-mapped host memory (cudaHostAlloc / torch pin_memory), at
 * least H + 3 * (stride + 4) bytes, 64-byte aligned (128 for line-aligned 128 B slots), H = 64 (128 for
 * 128 B slots), where stride = 288 for 288 B records, 192 for
 * 176 B compact slots (padded so that two slots cover three 128 B lines) and 128 for 128 B slots. Its first 64 bytes hold the
 * consumer index the producers read for backpressure; the rest is cap = floor((ring_bytes - H) /
 * (stride + 4)) slots followed by cap 4-byte commit tags (one per slot, written by the producer after its
 * record). A CUDA
 * device buffer instead (F2, on-GPU consumers) has no tag array: cap = floor((ring_bytes - 64) / 288).
 * nvbt_channel_bytes gives the ring_bytes that hold `slots` slots. */
size_t nvbt_channel_bytes(uint32_t record_bytes, uint64_t slots, int on_device);
/*
 * record_bytes: NVBT_RECORD_BYTES (288: every slot is an EM §5 record), NVBT_COMPACT_RECORD_BYTES (176:
 * base + 32-bit deltas, wide address sets as two slots; EM §5.1, F3) or NVBT_COMPACT128_RECORD_BYTES (128:
 * one whole PCIe line per record with base + 16-bit deltas, other records as three slots; EM §5.2). Every
 * way the drain delivers EM §5 records. One channel per context. The first open on a device loads every
 * workload kernel variant (cudaFuncGetAttributes): under CUDA lazy loading a kernel's first launch may
 * synchronise the context, which would wait for a producer that is itself waiting for the drain. A kernel
 * instrumented through include/nvbt_dev.cuh that traces must likewise be loaded (launched once, or
 * cudaFuncGetAttributes) before a producer of the same context can block on a full ring. */
#define NVBT_RECORD_BYTES 288
#define NVBT_COMPACT_RECORD_BYTES 176
#define NVBT_COMPACT128_RECORD_BYTES 128
int nvbt_channel_open(nvbt_ctx ctx, void* pinned_ring, size_t ring_bytes, uint32_t record_bytes,
                      nvbt_channel* out);
/* Called with a batch of n contiguous, fully written records (reserved field zeroed); return 0 to
 * continue, non-zero to stop draining (nvbt_channel_drain then returns NVBT_ESTATE). */
typedef int (*nvbt_drain_fn)(const void* records, uint64_t n_records, void* user);
/* Consumes records in ticket order until the context's stream is idle and every reserved record has
 * been delivered, or timeout_us elapses (-1 = no limit; NVBT_ETIMEDOUT). Producers reserve tickets in
 * per-warp blocks; tickets a block did not use (skip tag bit 31 for 288 B slots, 0xC0 skip slots for the
 * compact transports, EM §5) are consumed without being delivered. Runs on the calling thread,
 * concurrently with kernels already enqueued; it never synchronises the context's stream, so a drain
 * thread may run while another thread keeps enqueueing producers (it returns whenever it sees the stream
 * idle with everything delivered: call it again until the producer thread is done). *n_drained
 * (nullable) = records delivered by this call. A producer that waits 10 s (NVBT_PRODUCER_WAIT_MS, read at channel open) on a full ring gives up: its
 * record is dropped and counted (nvbt_channel_dropped), the drain then reports NVBT_ETIMEDOUT, and the
 * channel must be closed and reopened (the dropped ticket leaves a hole that is never committed). */
int nvbt_channel_drain(nvbt_channel ch, nvbt_drain_fn fn, void* user, int64_t timeout_us,
                       uint64_t* n_drained);
int nvbt_channel_close(nvbt_channel ch);
/* F2, on-GPU consumer ("can be analyzed directly on the GPU", P:L187 (§6.1)). A channel whose ring is
 * DEVICE memory (288 B records) is filled by the producers without backpressure: each SM takes slots
 * from its own 4096-slot chunk of the ring and each warp reserves the slots of the rest of its basic block
 * at once (x4 in loops), so some slots stay empty (the last chunk of every SM, a few per chunk and per
 * warp): size the ring for the records x 1.02 + 4096 x SMs slots; records that find no chunk are dropped
 * and counted. The ring
 * is analysed in place: per launch id first_launch + l, l < n_launches,
 *   out[3l + 0] = distinct 32 B sectors, out[3l + 1] = distinct 128 B lines over the lanes of E of all
 *   records of that launch (the launch's footprint, reading R-18), out[3l + 2] = records.
 * d_scratch: caller device memory of 4104 * table_slots + 8 * (3 * n_launches + 1) bytes, 16 B aligned
 * (an 8 B key and a 4 KB sector bitmap per slot); table_slots (a power of two) must exceed the number of
 * distinct (launch, 1 MB address region) pairs, ideally by 2x. n_launches <= 65536. EINVAL if a record's
 * launch id is outside the range or an address >= 2^48, or the table overflows (never hangs).
 * kernel_ms (nullable) = device time of the consumer kernels. Synchronises the context's stream.
 * Channels on pinned host memory return NVBT_ESTATE here; device channels return it from drain. */
int nvbt_trace_footprint(nvbt_channel ch, void* d_scratch, uint64_t table_slots, uint32_t first_launch,
                         uint32_t n_launches, uint64_t* out, float* kernel_ms);

/* Records the producers dropped after waiting 10 s (NVBT_PRODUCER_WAIT_MS) on a full ring (0 in a healthy run). */
int nvbt_channel_dropped(nvbt_channel ch, uint64_t* dropped);

/* Built-in drain callbacks. */
typedef struct { uint64_t n_rec, d1, d2; } nvbt_digest;         /* EM §5 multiset digest */
int nvbt_drain_digest(const void* records, uint64_t n_records, void* user /* nvbt_digest* */);
typedef struct { void* dst; uint64_t capacity; uint64_t n; } nvbt_copy_sink;   /* dst: host [capacity*288] */
int nvbt_drain_copy(const void* records, uint64_t n_records, void* user /* nvbt_copy_sink* */);
/* Counts and discards the records (user: nullable uint64_t* count): measures the transport alone. */
int nvbt_drain_discard(const void* records, uint64_t n_records, void* user /* uint64_t* */);
/* Host-side digest of an array of records (for checking copies). */
int nvbt_digest_records(const void* records, uint64_t n_records, nvbt_digest* out);
/* Decodes n_slots 176 B transport slots (EM §5.1; tags ignored) into EM §5 records at out (capacity
 * out_cap records); *n_out = records written. EINVAL on an unpaired wide slot or a too-small out. */
int nvbt_decode_compact(const void* slots, uint64_t n_slots, void* out, uint64_t out_cap, uint64_t* n_out);
/* The same for either compact transport: record_bytes NVBT_COMPACT_RECORD_BYTES or
 * NVBT_COMPACT128_RECORD_BYTES, slots packed record_bytes apart (tags ignored; 128 B skip slots, 0xC0 at
 * byte 27, carry no record, EM §5.2). EINVAL on a record whose continuation slots are missing or a too-small
 * out. */
int nvbt_decode_slots(const void* slots, uint64_t n_slots, uint32_t record_bytes, void* out, uint64_t out_cap,
                      uint64_t* n_out);

/* ---- trace-replay mode (a7; EM §3.5) ---- */
/* Writes events [first, first+n) of the counter-based generator (seed) as 16 B headers at d_hdr[n]
 * and, for memory pcs, 32 x u64 addresses at d_addr + 256*i. The context's program must be the
 * replay program (nvbt_program(NVBT_W_REPLAY, ...)). */
int nvbt_gen_events(nvbt_ctx ctx, uint64_t seed, uint64_t first, uint64_t n, void* d_hdr, void* d_addr);
/* Applies EM §2 items 1-4 to n events {u32 pc, warp, A, P} at d_hdr (slot i at d_addr + 256*i is read
 * only when kind(pc) is a memory kind and A&P != 0). pc >= n_pcs -> the event is ignored and counted
 * in the error word (nvbt_replay_errors). */
int nvbt_replay(nvbt_ctx ctx, const void* d_hdr, const void* d_addr, uint64_t n);
int nvbt_replay_errors(nvbt_ctx ctx, uint64_t* bad_events);

/* Staged replay: the same results as nvbt_replay (EM §2 items 1-4; north_star "trace-replay mode"),
 * computed in two passes per block of events. Pass A streams the headers (items 1-3) and lists each
 * executed memory event (E and a packed pc / tile / lane key: 8 B) in d_scratch; pass B streams the listed address slots
 * and computes S/L (item 4, P:L187-213 (§6.1)). d_scratch: caller-owned device memory, 256-byte aligned,
 * contents undefined between calls; a call processes n in blocks of as many events as the scratch holds.
 * Without NVBT_MEMDIV no list is written and d_scratch may be null. ENOMEM if scratch_bytes is below
 * nvbt_replay_scratch_size(ctx, 1). Asynchronous on the context's stream. */
int nvbt_replay_scratch_size(nvbt_ctx ctx, uint64_t max_events_per_block, size_t* bytes);
int nvbt_replay_staged(nvbt_ctx ctx, const void* d_hdr, const void* d_addr, uint64_t n, void* d_scratch,
                       size_t scratch_bytes);

/* ---- public device API (include/nvbt_dev.cuh): kernels outside the library instrument themselves ----
 * The compiled-in analogue of nvbit_insert_call / nvbit_add_call_arg (P:L123 (§4); Listing 8,
 * P:L243-246 (§6.1)): a kernel receives this POD by value and calls nvbt_on_instr / nvbt_on_bb /
 * nvbt_on_mem / nvbt_cta_flush at its injection points (pcs of the context's program table). Pointers
 * are device addresses inside the context's workspace (caller-owned, valid until nvbt_fini). */
#define NVBT_DEV_STATE_VERSION 1
typedef struct {
  uint32_t version;             /* NVBT_DEV_STATE_VERSION */
  uint32_t tools;               /* the tool set the hooks record: NVBT_TOOL_COUNT or NVBT_TOOL_BBCOUNT,
                                   and/or NVBT_TOOL_MEMDIV */
  unsigned long long* site;     /* per pc 4 u64 (t_issued, t_exec, w_issued, w_exec) at site + 4 pc, in
                                   each of `stripes` copies stripe_words apart (CTA c uses copy c % stripes) */
  unsigned long long* mem;      /* per pc 3 u64 (n, sectors, lines) at mem + 3 pc, striped the same way */
  unsigned long long* hist;     /* 66 u64 (hS[0..32], hL[0..32]), striped the same way */
  unsigned long long* per_warp; /* [2][n_warps] (executed thread / warp instructions) or NULL */
  uint64_t stripe_words;
  uint32_t stripes;             /* a power of two */
  uint32_t n_pcs;
  uint32_t n_warps;             /* per_warp length (0 without NVBT_PER_WARP) */
  uint32_t launch;              /* launch id this state was issued for (EM §5) */
} nvbt_dev_state;
/* Fills *out (pod_bytes must be sizeof(nvbt_dev_state)) for ONE instrumented launch of an external kernel
 * with `tools` (COUNT xor BBCOUNT, optionally MEMDIV; TRACE is not offered to external kernels: EINVAL);
 * takes the context's next launch id. ESTATE if a tool's flag was not enabled at init. Host-only. */
int nvbt_device_state(nvbt_ctx ctx, uint32_t tools, void* out_pod, size_t pod_bytes);

/* Number of kernels this context launched since init (for the bench's gpu_launches claim). */
int nvbt_launch_count(nvbt_ctx ctx, uint64_t* n);

#ifdef __cplusplus
}
#endif
#endif /* NVBT_H */
