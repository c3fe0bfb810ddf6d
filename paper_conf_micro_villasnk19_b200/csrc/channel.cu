// Device -> host trace channel (a6): a lock-free multi-producer ring in caller-pinned host memory.
//
// "NVBit allows one to ... collect reference addresses, which then can be analyzed directly on the GPU
// or sent to the CPU for further processing" (P:L187 (§6.1)). The paper gives no mechanism; this one:
//  * producers (warps, nvbt_dev.cuh emit<>) take a ticket t = atomicAdd(head, 1) in device memory, wait
//    while t >= tail + cap (tail = consumer index the host publishes in the ring's first 64 bytes, cached
//    in device memory), write the 288 B record (reserved field 0) into slot t % cap over PCIe with
//    coalesced stores, then a system-scope fence and a 4 B store of the tag (t / cap) + 1 into word t % cap
//    of a dense tag array that follows the slots (tags of neighbouring tickets share PCIe lines; a tag in
//    the record's own header line cost one extra partial-line write per record, see DESIGN §5 C4);
//  * the consumer (nvbt_channel_drain, calling thread) delivers slots in ticket order as soon as their tag
//    matches (a tag of an earlier lap never equals the current one, so tags are never cleared), calls the
//    user callback on contiguous batches and publishes tail.
#include <chrono>
#include <condition_variable>
#include <cstring>
#include <functional>
#include <sched.h>
#include <immintrin.h>
#include <thread>

#include <cstdlib>

#include "nvbt_internal.h"

struct nvbt_chan_s {
  nvbt_ctx ctx = nullptr;
  unsigned char* host = nullptr;      // ring base (host view)
  unsigned char* dev = nullptr;       // ring base (device view)
  unsigned char* slots = nullptr;     // host view of slot 0
  const uint32_t* tags = nullptr;     // host ring: host view of the tag array (cap words after the slots)
  uint64_t cap = 0;
  uint64_t consumed = 0;
  unsigned slot = 288;                 // bytes per ring slot (288 full, 176 compact)
  bool force_wide = false;
  unsigned long long wait_ns = 10000000000ull;   // a producer gives up after this long without room
  bool on_device = false;              // F2: ring in device memory, consumed by GPU kernels
  unsigned rstripes = 0;               // device ring: per-SM chunk stripes (see DevState)
  bool open = false;
  unsigned fmt = 0;                    // 0: 288 B records; 1: 176 B slots (EM §5.1); 2: 128 B slots (EM §5.2)
  size_t hdr = 64;                     // bytes before slot 0
  unsigned part_n = 0;                 // compact: slots of a multi-slot record seen at the ring end ...
  unsigned char part[3 * 192];         // ... stashed until the rest arrives as slots 0.. of the next lap
  std::vector<unsigned char> scratch;  // compact: decoded records of one batch
  // host rings: a private non-blocking stream for the drain's reads of the ticket counter. The drain never
  // synchronises the context's stream: another thread may be enqueueing producers on it, and waiting for
  // them would deadlock against the ring they are waiting on.
  cudaStream_t qs = nullptr;
  ~nvbt_chan_s() {
    if (qs) cudaStreamDestroy(qs);
  }
};

namespace nvbt {

static constexpr size_t HDR = 64;      // ring header (consumer index); 128 for 128 B slots so they are line aligned
static inline size_t hdr_of(uint32_t record_bytes) { return record_bytes == NVBT_COMPACT128_RECORD_BYTES ? 128 : HDR; }
static constexpr unsigned COMPACT_BYTES = NVBT_COMPACT_RECORD_BYTES;
// Ring stride of a compact slot: the 176 B slot padded to 192 B (pairs of slots cover 3 whole lines; PCIe
// D2H of SM stores, tools/peaks/d2h_pattern.cu: 176 B at a 176 B stride 33.0 GB/s of slot bytes, at a 192 B
// stride 36.5). The pad is never written or read.
static constexpr unsigned COMPACT_STRIDE = 192;
static constexpr unsigned SLOT128 = NVBT_COMPACT128_RECORD_BYTES;
static inline unsigned slot_stride(uint32_t record_bytes) { return record_bytes == COMPACT_BYTES ? COMPACT_STRIDE : record_bytes; }
static inline unsigned fmt_of(uint32_t record_bytes) { return record_bytes == COMPACT_BYTES ? 1u : record_bytes == SLOT128 ? 2u : 0u; }

void channel_state(nvbt_chan_s* ch, DevState* st) {
  st->ring = ch->dev + ch->hdr;
  st->tail = reinterpret_cast<const unsigned long long*>(ch->dev);
  st->cap = ch->cap;
  st->tags = ch->on_device ? nullptr : reinterpret_cast<unsigned*>(ch->dev + ch->hdr + ch->cap * ch->slot);
  st->slot_bytes = ch->slot;
  // compact = 1 / 3 (176 B / 128 B slots); 2 / 4 force the multi-slot form for every record
  // (NVBT_COMPACT_FORCE_WIDE=1, tests only)
  st->compact = ch->fmt == 1u ? (ch->force_wide ? 2u : 1u) : ch->fmt == 2u ? (ch->force_wide ? 4u : 3u) : 0u;
  st->no_wait = ch->on_device ? 1u : 0u;   // nobody frees device-ring slots: drop instead of waiting
  st->wait_ns = ch->wait_ns;
  st->rheads = ch->on_device ? ch->ctx->ctl + CTL_RHEAD : nullptr;
  st->rstripes = ch->rstripes;
}
bool channel_open(nvbt_chan_s* ch) { return ch && ch->open; }

// EM §5 digest constants and mix64 (splitmix64 output function).
static inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
struct DigestConsts {
  uint64_t c1[36], c2[36];
  DigestConsts() {
    for (int j = 0; j < 36; ++j) { c1[j] = mix64(0x1000 + j) | 1; c2[j] = mix64(0x2000 + j) | 1; }
  }
};
static const DigestConsts kDig;

static void digest_serial(const unsigned char* rec, uint64_t n, uint64_t* d1, uint64_t* d2) {
  uint64_t s1 = 0, s2 = 0;
  for (uint64_t r = 0; r < n; ++r) {
    uint64_t x[36];
    std::memcpy(x, rec + r * RECORD_BYTES, RECORD_BYTES);
    x[3] &= 0x00000000ffffffffull;  // bytes 28..31: EM §5 reserved, delivered as 0
    uint64_t h1 = 0, h2 = 0;
    for (int j = 0; j < 36; ++j) { h1 += x[j] * kDig.c1[j]; h2 += x[j] * kDig.c2[j]; }
    s1 += mix64(h1);
    s2 += mix64(h2);
  }
  *d1 += s1;
  *d2 += s2;
}

// Small persistent worker pool for host-side record processing (the drain's digest runs on all host
// cores: 362 GB of C4 records must be consumed at link speed). parallel_for splits [0, n) into equal
// contiguous parts, the calling thread takes part 0.
class Pool {
 public:
  static Pool& get() {
    static Pool p;
    return p;
  }
  unsigned size() const { return (unsigned)workers_.size() + 1; }
  void parallel_for(uint64_t n, const std::function<void(unsigned, uint64_t, uint64_t)>& fn) {
    const unsigned T = size();
    if (T == 1 || n < 4096) { fn(0, 0, n); return; }
    // one call at a time: the job slot (fn_, n_, pending_) is shared by the workers, so two drains on two
    // threads (or a digest during a drain) take turns instead of overwriting each other's job
    std::lock_guard<std::mutex> one(call_);
    {
      std::lock_guard<std::mutex> g(m_);
      fn_ = &fn; n_ = n; parts_ = T; pending_ = T - 1; ++gen_;
    }
    cv_.notify_all();
    fn(0, 0, n / T);
    std::unique_lock<std::mutex> lk(m_);
    done_.wait(lk, [&] { return pending_ == 0; });
    fn_ = nullptr;
  }
  ~Pool() {
    { std::lock_guard<std::mutex> g(m_); stop_ = true; ++gen_; }
    cv_.notify_all();
    for (auto& t : workers_) t.join();
  }

 private:
  Pool() {
    // one thread per CPU this process may run on (a rank bound to its GPU's NUMA node drains on that node's
    // cores only: drivers.bind_rank_to_gpu_numa), NVBT_DRAIN_THREADS overrides
    unsigned hw = std::thread::hardware_concurrency();
    cpu_set_t cs;
    CPU_ZERO(&cs);
    if (sched_getaffinity(0, sizeof cs, &cs) == 0 && CPU_COUNT(&cs) > 0) hw = (unsigned)CPU_COUNT(&cs);
    const char* e = getenv("NVBT_DRAIN_THREADS");
    if (e) hw = (unsigned)atoi(e);
    if (hw == 0) hw = 1;
    if (hw > 64) hw = 64;
    for (unsigned i = 1; i < hw; ++i) workers_.emplace_back([this, i] { run(i); });
  }
  void run(unsigned id) {
    uint64_t seen = 0;
    for (;;) {
      const std::function<void(unsigned, uint64_t, uint64_t)>* fn;
      uint64_t n;
      unsigned parts;
      {
        std::unique_lock<std::mutex> lk(m_);
        cv_.wait(lk, [&] { return stop_ || gen_ != seen; });
        if (stop_) return;
        seen = gen_;
        fn = fn_; n = n_; parts = parts_;
      }
      (*fn)(id, n * id / parts, n * (id + 1) / parts);
      {
        std::lock_guard<std::mutex> g(m_);
        if (--pending_ == 0) done_.notify_one();
      }
    }
  }
  std::vector<std::thread> workers_;
  std::mutex m_, call_;
  std::condition_variable cv_, done_;
  const std::function<void(unsigned, uint64_t, uint64_t)>* fn_ = nullptr;
  uint64_t n_ = 0, gen_ = 0;
  unsigned parts_ = 1, pending_ = 0;
  bool stop_ = false;
};

static void digest_range(const unsigned char* rec, uint64_t n, uint64_t* d1, uint64_t* d2) {
  if (n < 8192) { digest_serial(rec, n, d1, d2); return; }
  Pool& pool = Pool::get();
  std::vector<uint64_t> p1(pool.size(), 0), p2(pool.size(), 0);
  pool.parallel_for(n, [&](unsigned id, uint64_t lo, uint64_t hi) {
    digest_serial(rec + lo * RECORD_BYTES, hi - lo, &p1[id], &p2[id]);
  });
  for (size_t i = 0; i < p1.size(); ++i) { *d1 += p1[i]; *d2 += p2[i]; }
}


// Length of the prefix of slots [0, lim) whose tag equals `lap` (written and committed). Scans a short
// window serially and, when that is all ready, the rest of the batch in parallel on the pool.
// (bit 31 of a tag, kSkipTag, marks a ticket committed without a record: the unused rest of a producer's
// block of 288 B slots)
static inline bool slot_ready(const uint32_t* tag, uint32_t lap) {
  return (*reinterpret_cast<volatile const uint32_t*>(tag) & ~kSkipTag) == lap;
}
static uint64_t ready_prefix(const uint32_t* base, uint64_t lim, uint32_t lap) {
  const uint64_t w = std::min<uint64_t>(lim, 2048);
  uint64_t n = 0;
  while (n < w && slot_ready(base + n, lap)) ++n;
  if (n < w || n == lim) return n;
  Pool& pool = Pool::get();
  const uint64_t rest = lim - n;
  std::vector<uint64_t> first(pool.size(), UINT64_MAX);
  const uint32_t* b2 = base + n;
  pool.parallel_for(rest, [&](unsigned id, uint64_t lo, uint64_t hi) {
    uint64_t i = lo;
    while (i < hi && slot_ready(b2 + i, lap)) ++i;
    first[id] = i < hi ? i : UINT64_MAX;
  });
  uint64_t stop = rest;
  for (uint64_t f : first) stop = std::min(stop, f);
  return n + stop;
}
// ---- compact transport (EM §5.1): slot flags in byte 27 (kind | 0x80 compact, 0x40 / 0x20 wide halves;
// 0xC0 a skip slot of the 128 B transport: a ticket the producer's block did not use, EM §5.2)
static inline unsigned slot_flags(const unsigned char* sl) { return sl[27] & 0xE0u; }
static constexpr unsigned kSkipFlags = 0xC0u;
static inline bool starts_record(unsigned f) { return f != 0x20u && f != kSkipFlags; }

static void decode_compact_slot(const unsigned char* sl, unsigned char* out) {
  std::memcpy(out, sl, 28);
  out[27] = sl[27] & 0x1Fu;
  std::memset(out + 28, 0, 4);
  uint32_t A, P;
  std::memcpy(&A, sl + 16, 4);
  std::memcpy(&P, sl + 20, 4);
  const uint32_t E = A & P;
  uint64_t base;
  std::memcpy(&base, sl + 32, 8);
  for (int l = 0; l < 32; ++l) {
    int32_t d;
    std::memcpy(&d, sl + 48 + 4 * l, 4);
    const uint64_t a = ((E >> l) & 1u) ? base + (uint64_t)(int64_t)d : 0ull;
    std::memcpy(out + 32 + 8 * l, &a, 8);
  }
}
static void decode_wide_pair(const unsigned char* s0, const unsigned char* s1, unsigned char* out) {
  std::memcpy(out, s0, 28);
  out[27] = s0[27] & 0x1Fu;
  std::memset(out + 28, 0, 4);
  std::memcpy(out + 32, s0 + 32, 128);
  std::memcpy(out + 160, s1 + 32, 128);
}

// EM §5.2, 128 B slots: short (kind | 0x80): header, base at 32, 32 x i16 deltas at 40; long (kind | 0x40):
// three slots, lanes 0..11 at 32.. of the first, then per continuation slot (flag 0x20 at byte 27) 3 lanes
// at 0..23 and 12 lanes at 32..127.
static void decode_short128(const unsigned char* sl, unsigned char* out) {
  std::memcpy(out, sl, 28);
  out[27] = sl[27] & 0x1Fu;
  std::memset(out + 28, 0, 4);
  uint32_t A, P;
  std::memcpy(&A, sl + 16, 4);
  std::memcpy(&P, sl + 20, 4);
  const uint32_t E = A & P;
  uint64_t base;
  std::memcpy(&base, sl + 32, 8);
  for (int l = 0; l < 32; ++l) {
    int16_t d;
    std::memcpy(&d, sl + 40 + 2 * l, 2);
    const uint64_t a = ((E >> l) & 1u) ? base + (uint64_t)(int64_t)d : 0ull;
    std::memcpy(out + 32 + 8 * l, &a, 8);
  }
}
static void decode_long128(const unsigned char* s0, const unsigned char* s1, const unsigned char* s2, unsigned char* out) {
  std::memcpy(out, s0, 28);
  out[27] = s0[27] & 0x1Fu;
  std::memset(out + 28, 0, 4);
  std::memcpy(out + 32, s0 + 32, 96);             // lanes 0..11
  std::memcpy(out + 32 + 8 * 12, s1, 24);          // lanes 12..14
  std::memcpy(out + 32 + 8 * 15, s1 + 32, 96);     // lanes 15..26
  std::memcpy(out + 32 + 8 * 27, s2, 24);          // lanes 27..29
  std::memcpy(out + 32 + 8 * 30, s2 + 32, 16);     // lanes 30, 31
}
// slots per record starting with flags f (0x80 / none: 1; 0x40: 2 or 3)
static inline unsigned group_len(unsigned fmt, unsigned f) { return f == 0x40u ? (fmt == 2u ? 3u : 2u) : 1u; }
// the record whose first slot is s0 (its slots ss bytes apart)
static void decode_group(unsigned fmt, const unsigned char* s0, unsigned ss, unsigned char* out) {
  const unsigned f = slot_flags(s0);
  if (fmt == 2u) {
    if (f == 0x40u) decode_long128(s0, s0 + ss, s0 + 2 * ss, out);
    else decode_short128(s0, out);
  } else {
    if (f == 0x40u) decode_wide_pair(s0, s0 + ss, out);
    else decode_compact_slot(s0, out);
  }
}

// Decodes slots [0, n) into records; a wide-first at the end must not occur (caller keeps pairs whole).
// Parallel: count records per part, prefix, decode. Returns the record count.
static uint64_t decode_batch(const unsigned char* sl, uint64_t n, unsigned char* out, unsigned ss, unsigned fmt) {
  Pool& pool = Pool::get();
  std::vector<uint64_t> cnt(pool.size() + 1, 0), lo_of(pool.size(), 0), hi_of(pool.size(), 0);
  auto is_rec = [&](uint64_t i) { return starts_record(slot_flags(sl + (size_t)i * ss)); };
  pool.parallel_for(n, [&](unsigned id, uint64_t lo, uint64_t hi) {
    uint64_t c = 0;
    for (uint64_t i = lo; i < hi; ++i) c += is_rec(i);
    cnt[id + 1] = c;
    lo_of[id] = lo;
    hi_of[id] = hi;
  });
  for (size_t k = 1; k < cnt.size(); ++k) cnt[k] += cnt[k - 1];
  pool.parallel_for(n, [&](unsigned id, uint64_t lo, uint64_t hi) {
    uint64_t o = cnt[id];
    for (uint64_t i = lo; i < hi; ++i) {
      const unsigned char* s0 = sl + (size_t)i * ss;
      const unsigned f = slot_flags(s0);
      if (!starts_record(f)) continue;
      decode_group(fmt, s0, ss, out + (size_t)o * RECORD_BYTES);
      ++o;
    }
  });
  return cnt.back();
}

// Digest of the records encoded in slots [0, n) without materialising them (built-in digest callback).
static uint64_t digest_compact(const unsigned char* sl, uint64_t n, uint64_t* d1, uint64_t* d2, unsigned ss, unsigned fmt) {
  Pool& pool = Pool::get();
  std::vector<uint64_t> p1(pool.size(), 0), p2(pool.size(), 0), pc(pool.size(), 0);
  pool.parallel_for(n, [&](unsigned id, uint64_t lo, uint64_t hi) {
    alignas(16) unsigned char rec[RECORD_BYTES];
    uint64_t s1 = 0, s2 = 0, c = 0;
    for (uint64_t i = lo; i < hi; ++i) {
      const unsigned char* s0 = sl + (size_t)i * ss;
      const unsigned f = slot_flags(s0);
      if (!starts_record(f)) continue;
      decode_group(fmt, s0, ss, rec);
      digest_serial(rec, 1, &s1, &s2);
      ++c;
    }
    p1[id] = s1; p2[id] = s2; pc[id] = c;
  });
  uint64_t c = 0;
  for (size_t k = 0; k < p1.size(); ++k) { *d1 += p1[k]; *d2 += p2[k]; c += pc[k]; }
  return c;
}

}  // namespace nvbt

using namespace nvbt;

extern "C" {
int nvbt_drain_digest(const void* records, uint64_t n_records, void* user);
int nvbt_drain_copy(const void* records, uint64_t n_records, void* user);
int nvbt_drain_discard(const void* records, uint64_t n_records, void* user);
}

extern "C" {

size_t nvbt_channel_bytes(uint32_t record_bytes, uint64_t slots, int on_device) {
  return hdr_of(record_bytes) + slots * (slot_stride(record_bytes) + (on_device ? 0u : 4u));
}

int nvbt_channel_open(nvbt_ctx c, void* ring, size_t bytes, uint32_t record_bytes, nvbt_channel* out) {
  if (!c || !ring || !out) return set_error(NVBT_EINVAL, "null argument");
  if (!(c->flags & NVBT_TRACE)) return set_error(NVBT_ESTATE, "NVBT_TRACE not enabled at init");
  if (c->chan) return set_error(NVBT_ESTATE, "channel already open on this context");
  if (record_bytes != RECORD_BYTES && record_bytes != COMPACT_BYTES && record_bytes != SLOT128)
    return set_error(NVBT_EINVAL, "record_bytes %u is none of 288, 176, 128", record_bytes);
  if (reinterpret_cast<uintptr_t>(ring) % 64) return set_error(NVBT_EINVAL, "ring not 64-byte aligned");
  if (bytes < hdr_of(record_bytes) + 3 * (slot_stride(record_bytes) + 4))
    return set_error(NVBT_ENOMEM, "ring of %zu bytes holds < 3 slots", bytes);
  NVBT_CUDA(cudaSetDevice(c->device));
  { const int prc = preload_workload_kernels(c->device); if (prc) return prc; }
  cudaPointerAttributes pa{};
  NVBT_CUDA(cudaPointerGetAttributes(&pa, ring));
  const bool on_device = pa.type == cudaMemoryTypeDevice;
  if (!on_device && (pa.type != cudaMemoryTypeHost || pa.devicePointer == nullptr))
    return set_error(NVBT_EINVAL, "ring is neither pinned device-mapped host memory nor device memory");
  if (on_device && record_bytes != RECORD_BYTES)
    return set_error(NVBT_EINVAL, "device-memory channels use 288 B records");
  auto* ch = new (std::nothrow) nvbt_chan_s();
  if (!ch) return set_error(NVBT_ENOMEM, "host allocation failed");
  ch->ctx = c;
  ch->on_device = on_device;
  ch->host = on_device ? nullptr : static_cast<unsigned char*>(ring);
  ch->dev = static_cast<unsigned char*>(on_device ? ring : pa.devicePointer);
  ch->hdr = hdr_of(record_bytes);
  ch->slots = on_device ? nullptr : ch->host + ch->hdr;
  ch->slot = slot_stride(record_bytes);
  ch->fmt = fmt_of(record_bytes);
  { const char* e = getenv("NVBT_COMPACT_FORCE_WIDE"); ch->force_wide = e && atoi(e) != 0; }
  { const char* e = getenv("NVBT_PRODUCER_WAIT_MS"); if (e && atoll(e) > 0) ch->wait_ns = 1000000ull * (unsigned long long)atoll(e); }
  // host rings: each slot has a 4 B tag in the array after the slots; device rings carry the tag in-record
  ch->cap = (bytes - ch->hdr) / (ch->slot + (on_device ? 0u : 4u));
  ch->tags = on_device ? nullptr : reinterpret_cast<const uint32_t*>(ch->host + ch->hdr + ch->cap * ch->slot);
  if (on_device) {
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device);
    ch->rstripes = std::min<unsigned>((unsigned)sms, kMaxRingStripes);
  }
  cudaError_t e = cudaSuccess;
  if (on_device) e = cudaMemsetAsync(ring, 0, HDR + ch->cap * record_bytes, c->stream);
  else std::memset(ch->host, 0, ch->hdr + ch->cap * (ch->slot + 4));
  if (on_device && e == cudaSuccess) {   // every stripe starts without a chunk; chunk counter 0
    std::vector<unsigned long long> w(ch->rstripes + 1, ((unsigned long long)kRingNoChunk << 32) | kRingChunk);
    w.back() = 0;
    e = cudaMemcpyAsync(c->ctl + CTL_RHEAD, w.data(), w.size() * 8, cudaMemcpyHostToDevice, c->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);   // w is a host temporary
  }
  if (e == cudaSuccess) e = cudaMemsetAsync(c->ctl + CTL_HEAD, 0, 3 * 8, c->stream);  // head, tail_cache, dropped
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
  if (e == cudaSuccess && !on_device) e = cudaStreamCreateWithFlags(&ch->qs, cudaStreamNonBlocking);
  if (e != cudaSuccess) { delete ch; return set_error(NVBT_ECUDA, "channel reset: %s", cudaGetErrorString(e)); }
  ch->open = true;
  c->chan = ch;
  *out = ch;
  return NVBT_OK;
}

// ---- F2: on-GPU consumer of a device-memory channel ---------------------------------------------
// Footprint of the recorded accesses per launch: distinct 32 B sectors and 128 B lines over the lanes of
// E. The set is a sparse bitmap: an open-addressing table of 1 MB regions keyed (launch, addr >> 20),
// each owning a 4 KB block of 4 sector bits per line (8192 lines). The blocks cost 1/256 of the address
// span a launch touches and stay L2-resident, so the kernel streams the records from HBM once.
namespace nvbt {
constexpr unsigned long long kFpEmpty = ~0ull;
constexpr int kFpRegionShift = 20;           // 1 MB regions
constexpr unsigned kFpWords = (1u << (kFpRegionShift - 7)) / 8;   // 32-bit words per block (8 lines each)

__device__ __forceinline__ unsigned nib_nonzero(unsigned x) { return (x | x >> 1 | x >> 2 | x >> 3) & 0x11111111u; }

// Table slot of region key k (warp-uniform call: every lane probes the same addresses). Two-entry cache
// (c0 most recent). Returns false if the table is full.
__device__ __forceinline__ bool fp_slot(unsigned long long k, unsigned long long* __restrict__ keys,
                                        unsigned long long mask, unsigned long long (&ck)[2],
                                        unsigned long long (&cs)[2], unsigned long long& slot) {
  if (k == ck[0]) { slot = cs[0]; return true; }
  if (k == ck[1]) {
    slot = cs[1];
    ck[1] = ck[0]; cs[1] = cs[0]; ck[0] = k; cs[0] = slot;
    return true;
  }
  unsigned long long h = ((k * 0x9E3779B97F4A7C15ull) >> 24) & mask;
  for (unsigned long long probes = 0; probes <= mask; ++probes) {   // bounded: a full table is an error
    // lane 0 reads and claims; the warp follows its view (lanes reading on their own could disagree
    // while another warp inserts)
    unsigned long long v = 0;
    if (lane_id() == 0) {
      v = *reinterpret_cast<volatile unsigned long long*>(keys + h);
      if (v == kFpEmpty) v = atomicCAS(keys + h, kFpEmpty, k);
    }
    v = __shfl_sync(0xffffffffu, v, 0);
    if (v == kFpEmpty || v == k) {
      ck[1] = ck[0]; cs[1] = cs[0]; ck[0] = k; cs[0] = h;
      slot = h;
      return true;
    }
    h = (h + 1) & mask;
  }
  return false;
}

// Per-lane table lookup (divergent callers: each quad leader looks up its own record's region), with a
// per-lane two-entry cache. Returns false if the table is full.
__device__ __forceinline__ bool fp_slot_lane(unsigned long long k, unsigned long long* __restrict__ keys,
                                             unsigned long long mask, unsigned long long (&ck)[2],
                                             unsigned long long (&cs)[2], unsigned long long& slot) {
  if (k == ck[0]) { slot = cs[0]; return true; }
  if (k == ck[1]) {
    slot = cs[1];
    ck[1] = ck[0]; cs[1] = cs[0]; ck[0] = k; cs[0] = slot;
    return true;
  }
  unsigned long long h = ((k * 0x9E3779B97F4A7C15ull) >> 24) & mask;
  for (unsigned long long probes = 0; probes <= mask; ++probes) {
    unsigned long long v = *reinterpret_cast<volatile unsigned long long*>(keys + h);
    if (v == kFpEmpty) v = atomicCAS(keys + h, kFpEmpty, k);
    if (v == kFpEmpty || v == k) {
      ck[1] = ck[0]; cs[1] = cs[0]; ck[0] = k; cs[0] = h;
      slot = h;
      return true;
    }
    h = (h + 1) & mask;
  }
  return false;
}

// One record (warp-uniform control flow): for each distinct (region, word) among the lanes of E, OR
// the lanes' sector bits into the region's block with one fire-and-forget reduction; distinct counts come
// from k_fp_count afterwards.
__device__ __forceinline__ void fp_record(unsigned launch, unsigned E, unsigned long long a, unsigned lane,
                                          unsigned long long* __restrict__ keys, unsigned* __restrict__ pool,
                                          unsigned long long mask, unsigned long long* err,
                                          unsigned long long (&ck)[2], unsigned long long (&cs)[2]) {
  bool on = (E >> lane) & 1u;
  if (on && (a >> 48)) { atomicAdd(err, 1ull); on = false; }
  const unsigned long long rkey = ((unsigned long long)launch << (48 - kFpRegionShift)) | (a >> kFpRegionShift);
  const unsigned line = (unsigned)(a >> 7) & (8 * kFpWords - 1);
  const unsigned word = line >> 3;
  const unsigned bits = 1u << ((line & 7) * 4 + ((unsigned)(a >> 5) & 3));
  unsigned pend = __ballot_sync(0xffffffffu, on);
  if (pend == 0) return;
  while (pend) {
    const unsigned f = __ffs(pend) - 1;
    const unsigned long long k = __shfl_sync(0xffffffffu, rkey, f);
    const unsigned wd = __shfl_sync(0xffffffffu, word, f);
    const bool mine = on && rkey == k && word == wd;
    const unsigned m = __ballot_sync(0xffffffffu, mine);
    const unsigned v = __reduce_or_sync(0xffffffffu, mine ? bits : 0u);
    pend &= ~m;
    on = on && !mine;
    unsigned long long slot;
    if (!fp_slot(k, keys, mask, ck, cs, slot)) { if (lane == f) atomicAdd(err, 1ull); continue; }
    if (lane == f) atomicOr(pool + slot * kFpWords + wd, v);
  }
}

// Distinct counts per launch from the region blocks: sectors = set bits, lines = non-zero nibbles.
// One warp per table slot; per-CTA shared bins when n_launches is small.
__global__ void __launch_bounds__(256) k_fp_count(const unsigned long long* __restrict__ keys,
                                                   const unsigned* __restrict__ pool, unsigned long long slots,
                                                   unsigned long long* __restrict__ counts, unsigned n_launches) {
  constexpr unsigned kBins = 1024;
  __shared__ unsigned long long bins[2 * kBins];
  const bool shared = n_launches <= kBins;
  if (shared)
    for (unsigned i = threadIdx.x; i < 2 * n_launches; i += blockDim.x) bins[i] = 0;
  __syncthreads();
  const unsigned lane = lane_id();
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  for (unsigned long long sl = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5; sl < slots; sl += warps) {
    const unsigned long long k = keys[sl];
    if (k == kFpEmpty) continue;
    unsigned ns = 0, nl = 0;
    const uint4* blk = reinterpret_cast<const uint4*>(pool + sl * kFpWords);
    for (unsigned i = lane; i < kFpWords / 4; i += 32) {
      const uint4 v = blk[i];
      ns += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
      nl += __popc(nib_nonzero(v.x)) + __popc(nib_nonzero(v.y)) + __popc(nib_nonzero(v.z)) + __popc(nib_nonzero(v.w));
    }
    ns = __reduce_add_sync(0xffffffffu, ns);
    nl = __reduce_add_sync(0xffffffffu, nl);
    if (lane == 0) {
      const unsigned l = (unsigned)(k >> (48 - kFpRegionShift));
      if (shared) { atomicAdd(bins + 2 * l, (unsigned long long)ns); atomicAdd(bins + 2 * l + 1, (unsigned long long)nl); }
      else { atomicAdd(counts + 3ull * l, (unsigned long long)ns); atomicAdd(counts + 3ull * l + 1, (unsigned long long)nl); }
    }
  }
  if (shared) {
    __syncthreads();
    for (unsigned i = threadIdx.x; i < 2 * n_launches; i += blockDim.x)
      if (bins[i]) atomicAdd(counts + 3ull * (i >> 1) + (i & 1), bins[i]);
  }
}

// Committed slots lie in the chunks handed out so far, [0, min(chunks * kRingChunk, cap)); slots never
// written (the unused tail of each SM's last chunk, slots a warp reserved but did not use) have tag 0 and
// are skipped. Each warp takes a contiguous range of slots, 32 at a time: lane i reads record i's
// header, then the warp walks the 32 records 8 at a time, 4 lanes per record (quad pass).
__global__ void __launch_bounds__(256, 4) k_footprint(const unsigned char* __restrict__ ring,
                                                    const unsigned long long* __restrict__ chunks,
                                                    unsigned long long cap,
                                                    unsigned long long* __restrict__ keys, unsigned* __restrict__ pool,
                                                    unsigned long long mask, unsigned long long* __restrict__ counts,
                                                    unsigned first, unsigned n_launches) {
  const unsigned lane = lane_id();
  const unsigned long long n_slots = *chunks * kRingChunk < cap ? *chunks * kRingChunk : cap;
  const unsigned long long warps = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  const unsigned long long w = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
  const unsigned long long per = (n_slots + warps - 1) / warps;
  const unsigned long long r0 = w * per, r1 = r0 + per < n_slots ? r0 + per : n_slots;
  unsigned long long* err = counts + 3ull * n_launches;
  unsigned cur = 0xFFFFFFFFu;
  unsigned long long nrec = 0;
  unsigned long long ck[2] = {kFpEmpty, kFpEmpty}, cs[2] = {0, 0};
  // headers are loaded one 32-record group ahead
  uint4 nh1 = make_uint4(0, 0, 0, 0);
  unsigned nl = 0;
  if (r0 + lane < r1) {
    const unsigned char* rec = ring + 64 + (r0 + lane) * RECORD_BYTES;
    nh1 = __ldg(reinterpret_cast<const uint4*>(rec + 16));   // A P op|w|k tag
    nl = __ldg(reinterpret_cast<const unsigned*>(rec));
  }
  for (unsigned long long base = r0; base < r1; base += 32) {
    const unsigned cnt = r1 - base < 32 ? (unsigned)(r1 - base) : 32u;
    unsigned lid = 0xFFFFFFFFu, E = 0;
    if (lane < cnt && nh1.w == 1u) { lid = nl - first; E = nh1.x & nh1.y; }
    nh1 = make_uint4(0, 0, 0, 0);
    if (base + 32 + lane < r1) {
      const unsigned char* rec = ring + 64 + (base + 32 + lane) * RECORD_BYTES;
      nh1 = __ldg(reinterpret_cast<const uint4*>(rec + 16));
      nl = __ldg(reinterpret_cast<const unsigned*>(rec));
    }
    const bool ok = lid < n_launches;
    const unsigned bad = __ballot_sync(0xffffffffu, lid != 0xFFFFFFFFu && !ok);
    if (bad) { if (lane == 0) atomicAdd(err, (unsigned long long)__popc(bad)); E = ok ? E : 0u; }
    const unsigned okm = __ballot_sync(0xffffffffu, ok);
    if (okm) {   // record counts: a warp's range nearly always holds one launch
      const unsigned l0 = __shfl_sync(0xffffffffu, lid, __ffs(okm) - 1);
      if (__all_sync(0xffffffffu, !ok || lid == l0)) {
        if (l0 != cur) {
          if (lane == 0 && cur != 0xFFFFFFFFu) atomicAdd(counts + 3ull * cur + 2, nrec);
          cur = l0; nrec = 0;
        }
        nrec += __popc(okm);
      } else {
        unsigned pend = okm;
        while (pend) {
          const unsigned l = __shfl_sync(0xffffffffu, lid, __ffs(pend) - 1);
          const unsigned m = __ballot_sync(0xffffffffu, ok && lid == l);
          if (lane == 0) atomicAdd(counts + 3ull * l + 2, (unsigned long long)__popc(m));
          pend &= ~m;
        }
      }
    }
    const unsigned live = __ballot_sync(0xffffffffu, ok && E != 0u);
    // quad pass, 8 records at a time: lanes 4b..4b+3 read record j+b's 32 addresses (8 each, 4 x 16 B)
    // and check that all lanes of E fall in one 1 KB word of one region; if so the quad's first lane ORs
    // the record's sector bits with one atomic (common: a warp access covers <= 1 KB). Records spanning
    // several words take the warp-cooperative fp_record().
    const unsigned qb = lane >> 2, qq = lane & 3u;
    for (unsigned j = 0; j < 32; j += 8) {
      if (((live >> j) & 0xFFu) == 0u) continue;   // uniform
      const unsigned jj = j + qb;
      const bool qlive = (live >> jj) & 1u;
      const unsigned qE = __shfl_sync(0xffffffffu, E, jj) >> (8u * qq);
      const unsigned ql = __shfl_sync(0xffffffffu, lid, jj);
      // per lane: the first active address is the reference; every active address must lie in the
      // reference's 1 KB word (same a >> 10); sector bit = (a >> 5) & 31 within that word
      unsigned ref_lo = 0, ref_hi = 0, nd = 0, bits = 0;
      bool have = false;
      if (qlive) {
        const uint4* src = reinterpret_cast<const uint4*>(ring + 64 + (base + jj) * RECORD_BYTES + 32 + 64 * qq);
        uint4 va[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) va[k] = __ldcs(src + k);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
#pragma unroll
          for (int t = 0; t < 2; ++t) {
            const bool act = (qE >> (2 * k + t)) & 1u;
            const unsigned lo = t ? va[k].z : va[k].x, hi = t ? va[k].w : va[k].y;
            const bool first = act && !have;
            ref_lo = first ? lo : ref_lo;
            ref_hi = first ? hi : ref_hi;
            have = have || act;
            nd |= act ? (((lo ^ ref_lo) >> 10) | (hi ^ ref_hi)) : 0u;
            bits |= act ? 1u << ((lo >> 5) & 31u) : 0u;
          }
        }
      }
      // quad reduction: one 1 KB word (below 2^48) for the whole record?
      bool same = nd == 0u && (ref_hi >> 16) == 0u;
#pragma unroll
      for (unsigned d = 1; d <= 2; d <<= 1) {
        const unsigned oh = __shfl_xor_sync(0xffffffffu, (unsigned)have, d);
        const unsigned olo = __shfl_xor_sync(0xffffffffu, ref_lo, d);
        const unsigned ohi = __shfl_xor_sync(0xffffffffu, ref_hi, d);
        const unsigned ob = __shfl_xor_sync(0xffffffffu, bits, d);
        const unsigned os = __shfl_xor_sync(0xffffffffu, (unsigned)same, d);
        same = same && os != 0u && (!have || !oh || (((olo ^ ref_lo) >> 10) | (ohi ^ ref_hi)) == 0u);
        if (!have && oh) { ref_lo = olo; ref_hi = ohi; }
        have = have || oh != 0u;
        bits |= ob;
      }
      const unsigned long long key =
          ((unsigned long long)ql << (48 - kFpRegionShift)) | ((((unsigned long long)ref_hi << 32) | ref_lo) >> kFpRegionShift);
      const unsigned wd = (ref_lo >> 10) & (kFpWords - 1u);
      if (qlive && same && qq == 0) {
        unsigned long long slot;
        if (fp_slot_lane(key, keys, mask, ck, cs, slot)) atomicOr(pool + slot * kFpWords + wd, bits);
        else atomicAdd(err, 1ull);
      }
      unsigned slow = __ballot_sync(0xffffffffu, qlive && !same && qq == 0);
      while (slow) {
        const unsigned b = (__ffs(slow) - 1) >> 2;
        slow &= slow - 1;
        const unsigned r = j + b;
        const unsigned long long a = __ldcs(reinterpret_cast<const unsigned long long*>(ring + 64 + (base + r) * RECORD_BYTES + 32) + lane);
        unsigned long long wck[2] = {kFpEmpty, kFpEmpty}, wcs[2] = {0, 0};
        fp_record(__shfl_sync(0xffffffffu, lid, r), __shfl_sync(0xffffffffu, E, r), a, lane, keys, pool, mask, err, wck, wcs);
      }
    }
  }
  if (lane == 0 && cur != 0xFFFFFFFFu) atomicAdd(counts + 3ull * cur + 2, nrec);
}
}  // namespace nvbt

int nvbt_trace_footprint(nvbt_channel ch, void* d_scratch, uint64_t table_slots, uint32_t first_launch,
                         uint32_t n_launches, uint64_t* out, float* kernel_ms) {
  if (!ch || !d_scratch || !out || n_launches == 0) return set_error(NVBT_EINVAL, "null argument");
  if (!ch->on_device) return set_error(NVBT_ESTATE, "footprint needs a device-memory channel");
  if (table_slots == 0 || (table_slots & (table_slots - 1))) return set_error(NVBT_EINVAL, "table_slots must be a power of two");
  if (n_launches > (1u << 16)) return set_error(NVBT_EINVAL, "n_launches > 65536");
  nvbt_ctx c = ch->ctx;
  NVBT_CUDA(cudaSetDevice(c->device));
  if (reinterpret_cast<uintptr_t>(d_scratch) % 16) return set_error(NVBT_EINVAL, "d_scratch not 16-byte aligned");
  // [blocks: 4 KB per slot][keys: 8 B per slot][counts]
  auto* pool = static_cast<unsigned*>(d_scratch);
  auto* keys = reinterpret_cast<unsigned long long*>(pool + table_slots * kFpWords);
  unsigned long long* counts = keys + table_slots;
  NVBT_CUDA(cudaMemsetAsync(keys, 0xff, table_slots * 8, c->stream));
  NVBT_CUDA(cudaMemsetAsync(pool, 0, table_slots * kFpWords * 4, c->stream));
  NVBT_CUDA(cudaMemsetAsync(counts, 0, (3ull * n_launches + 1) * 8, c->stream));
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device);
  cudaEvent_t ev[2] = {nullptr, nullptr};
  if (kernel_ms) { NVBT_CUDA(cudaEventCreate(&ev[0])); NVBT_CUDA(cudaEventCreate(&ev[1])); cudaEventRecord(ev[0], c->stream); }
  k_footprint<<<sms * 8, 256, 0, c->stream>>>(ch->dev, c->ctl + CTL_RHEAD + ch->rstripes, ch->cap, keys, pool,
                                              table_slots - 1, counts, first_launch, n_launches);
  NVBT_CUDA(cudaGetLastError());
  k_fp_count<<<(unsigned)std::min<unsigned long long>((table_slots + 7) / 8, (unsigned long long)sms * 8), 256, 0,
               c->stream>>>(keys, pool, table_slots, counts, n_launches);
  NVBT_CUDA(cudaGetLastError());
  c->launches += 2;
  if (kernel_ms) {
    cudaEventRecord(ev[1], c->stream);
    cudaEventSynchronize(ev[1]);
    cudaEventElapsedTime(kernel_ms, ev[0], ev[1]);
    cudaEventDestroy(ev[0]); cudaEventDestroy(ev[1]);
  }
  std::vector<unsigned long long> h(3ull * n_launches + 1);
  NVBT_CUDA(cudaMemcpyAsync(h.data(), counts, h.size() * 8, cudaMemcpyDeviceToHost, c->stream));
  NVBT_CUDA(cudaStreamSynchronize(c->stream));
  if (h.back()) return set_error(NVBT_EINVAL, "%llu records out of range (launch id or address >= 2^48) or table_slots too small", h.back());
  std::memcpy(out, h.data(), 3ull * n_launches * 8);
  return NVBT_OK;
}

int nvbt_channel_close(nvbt_channel ch) {
  if (!ch) return set_error(NVBT_EINVAL, "channel is null");
  if (ch->ctx && ch->ctx->chan == ch) ch->ctx->chan = nullptr;
  delete ch;
  return NVBT_OK;
}

int nvbt_channel_dropped(nvbt_channel ch, uint64_t* dropped) {
  if (!ch || !dropped) return set_error(NVBT_EINVAL, "null argument");
  nvbt_ctx c = ch->ctx;
  NVBT_CUDA(cudaMemcpyAsync(dropped, c->ctl + CTL_DROPPED, 8, cudaMemcpyDeviceToHost, c->stream));
  NVBT_CUDA(cudaStreamSynchronize(c->stream));
  return NVBT_OK;
}

int nvbt_channel_drain(nvbt_channel ch, nvbt_drain_fn fn, void* user, int64_t timeout_us, uint64_t* n_drained) {
  if (!ch || !fn) return set_error(NVBT_EINVAL, "null argument");
  if (!ch->open) return set_error(NVBT_ESTATE, "channel not open");
  if (ch->on_device) return set_error(NVBT_ESTATE, "device-memory channel: use the GPU consumers (nvbt_trace_footprint)");
  nvbt_ctx c = ch->ctx;
  NVBT_CUDA(cudaSetDevice(c->device));
  const auto t0 = std::chrono::steady_clock::now();
  const uint64_t kBatch = 1u << 17;
  volatile uint64_t* tail = reinterpret_cast<volatile uint64_t*>(ch->host);
  uint64_t delivered = 0;
  int rc = NVBT_OK;
  for (;;) {
    const uint64_t slot = ch->consumed % ch->cap;
    const uint32_t lap = static_cast<uint32_t>(ch->consumed / ch->cap) + 1u;
    const uint64_t lim = std::min<uint64_t>(ch->cap - slot, kBatch);
    const unsigned sb = ch->slot;
    const uint64_t n = ready_prefix(ch->tags + slot, lim, lap);
    if (n && sb == RECORD_BYTES) {
      std::atomic_thread_fence(std::memory_order_acquire);
      unsigned char* base = ch->slots + slot * RECORD_BYTES;
      // runs of records between skip tickets (tags with kSkipTag carry no record)
      const uint32_t* tg = ch->tags + slot;
      int urc = 0;
      for (uint64_t i = 0; i < n && !urc;) {
        uint64_t j = i;
        while (j < n && !(tg[j] & kSkipTag)) ++j;
        if (j > i) {
          urc = fn(base + i * RECORD_BYTES, j - i, user);
          delivered += j - i;
        }
        i = j;
        while (i < n && (tg[i] & kSkipTag)) ++i;
      }
      ch->consumed += n;
      std::atomic_thread_fence(std::memory_order_release);
      *tail = ch->consumed;
      if (urc) { rc = set_error(NVBT_ESTATE, "drain callback returned %d", urc); break; }
      continue;
    }
    if (n) {  // compact transports: decode slots into EM §5 records, keep multi-slot records together
      std::atomic_thread_fence(std::memory_order_acquire);
      const unsigned char* base = ch->slots + slot * sb;
      if (ch->scratch.size() < (kBatch + 1) * RECORD_BYTES) ch->scratch.resize((kBatch + 1) * RECORD_BYTES);
      unsigned char* out = ch->scratch.data();
      uint64_t first = 0, end = n, consume = n, o = 0;
      if (ch->part_n) {   // the rest of a record stashed at the ring end: its continuation slots come first
        const unsigned g = group_len(ch->fmt, slot_flags(ch->part));
        const uint64_t k = std::min<uint64_t>(g - ch->part_n, n);
        bool bad = false;
        for (uint64_t i = 0; i < k; ++i) bad |= slot_flags(base + i * sb) != 0x20u;
        if (bad) { rc = set_error(NVBT_ESTATE, "channel: multi-slot record without its continuation"); break; }
        for (uint64_t i = 0; i < k; ++i) std::memcpy(ch->part + (ch->part_n + i) * sb, base + i * sb, sb);
        ch->part_n += (unsigned)k;
        first = k;
        if (ch->part_n == g) {
          decode_group(ch->fmt, ch->part, sb, out);
          ch->part_n = 0;
          o = 1;
        }
      }
      // a record whose slots are not all ready (or continue in the next lap) ends the batch early
      uint64_t cut = end;
      const unsigned glong = ch->fmt == 2u ? 3u : 2u;
      for (uint64_t back = 1; back < glong && back <= end - first; ++back)
        if (slot_flags(base + (end - back) * sb) == 0x40u) { cut = end - back; break; }
      if (cut < end) {
        if (slot + end == ch->cap) {      // continues in slots 0.. of the next lap: stash what is here
          std::memcpy(ch->part, base + cut * sb, (end - cut) * sb);
          ch->part_n = (unsigned)(end - cut);
        } else {
          consume = cut;                   // the rest is not ready yet: take the record next time
        }
        end = cut;
      }
      int urc = 0;
      if (fn == nvbt_drain_digest && user) {   // fused decode + digest, no staging of records
        auto* dg = static_cast<nvbt_digest*>(user);
        if (o) urc = fn(out, o, user);
        const uint64_t k = digest_compact(base + first * sb, end - first, &dg->d1, &dg->d2, sb, ch->fmt);
        dg->n_rec += k;
        o += k;
      } else {
        o += decode_batch(base + first * sb, end - first, out + o * RECORD_BYTES, sb, ch->fmt);
        urc = o ? fn(out, o, user) : 0;
      }
      ch->consumed += consume;
      delivered += o;
      std::atomic_thread_fence(std::memory_order_release);
      *tail = ch->consumed;
      if (urc) { rc = set_error(NVBT_ESTATE, "drain callback returned %d", urc); break; }
      if (consume) continue;
    }
    const cudaError_t q = cudaStreamQuery(c->stream);
    if (q == cudaSuccess) {
      // the producers enqueued before the query have finished, so head is final for them (read on the
      // channel's own stream: never wait on the context's stream, see nvbt_chan_s::qs)
      uint64_t ctl[3];
      NVBT_CUDA(cudaMemcpyAsync(ctl, c->ctl + CTL_HEAD, sizeof ctl, cudaMemcpyDeviceToHost, ch->qs));
      NVBT_CUDA(cudaStreamSynchronize(ch->qs));
      if (ch->consumed >= ctl[0]) break;  // every ticket handed out has been delivered
      if (ctl[2] != 0) {
        rc = set_error(NVBT_ETIMEDOUT, "%llu records dropped by producers (ring full, no consumer)",
                       (unsigned long long)ctl[2]);
        break;
      }
    } else if (q != cudaErrorNotReady) {
      rc = set_error(NVBT_ECUDA, "stream error: %s", cudaGetErrorString(q));
      break;
    }
    if (timeout_us >= 0) {
      const auto us = std::chrono::duration_cast<std::chrono::microseconds>(std::chrono::steady_clock::now() - t0).count();
      if (us > timeout_us) { rc = set_error(NVBT_ETIMEDOUT, "drain timed out after %lld us", (long long)us); break; }
    }
    for (int i = 0; i < 64; ++i) _mm_pause();
  }
  if (n_drained) *n_drained = delivered;
  return rc;
}

int nvbt_drain_discard(const void*, uint64_t n, void* user) {
  if (user) *static_cast<uint64_t*>(user) += n;
  return 0;
}

int nvbt_drain_digest(const void* records, uint64_t n, void* user) {
  auto* d = static_cast<nvbt_digest*>(user);
  if (!d) return 1;
  digest_range(static_cast<const unsigned char*>(records), n, &d->d1, &d->d2);
  d->n_rec += n;
  return 0;
}

int nvbt_drain_copy(const void* records, uint64_t n, void* user) {
  auto* s = static_cast<nvbt_copy_sink*>(user);
  if (!s || s->n + n > s->capacity) return 1;
  unsigned char* dst = static_cast<unsigned char*>(s->dst) + s->n * RECORD_BYTES;
  const unsigned char* src = static_cast<const unsigned char*>(records);
  Pool::get().parallel_for(n, [&](unsigned, uint64_t lo, uint64_t hi) {
    std::memcpy(dst + lo * RECORD_BYTES, src + lo * RECORD_BYTES, (hi - lo) * RECORD_BYTES);
    for (uint64_t r = lo; r < hi; ++r) std::memset(dst + r * RECORD_BYTES + 28, 0, 4);
  });
  s->n += n;
  return 0;
}

int nvbt_decode_slots(const void* slots, uint64_t n, uint32_t record_bytes, void* out, uint64_t cap, uint64_t* n_out) {
  if ((!slots && n) || (!out && cap) || !n_out) return set_error(NVBT_EINVAL, "null argument");
  const unsigned fmt = fmt_of(record_bytes);
  if (fmt == 0u) return set_error(NVBT_EINVAL, "record_bytes %u is not a compact transport (176 or 128)", record_bytes);
  const unsigned ss = record_bytes;   // slots packed back to back (no ring padding)
  const unsigned char* sl = static_cast<const unsigned char*>(slots);
  unsigned char* o = static_cast<unsigned char*>(out);
  uint64_t k = 0;
  for (uint64_t i = 0; i < n;) {
    const unsigned char* s0 = sl + i * ss;
    const unsigned f = slot_flags(s0);
    if (f == kSkipFlags) { ++i; continue; }   // an unused ticket of a producer's block
    if (f != 0x80u && f != 0x40u)
      return set_error(NVBT_EINVAL, "slot %llu: not the first slot of a record (flags 0x%x)", (unsigned long long)i, f);
    const unsigned g = group_len(fmt, f);
    if (i + g > n) return set_error(NVBT_EINVAL, "slot %llu: record continues past the last slot", (unsigned long long)i);
    for (unsigned q = 1; q < g; ++q)
      if (slot_flags(s0 + q * ss) != 0x20u)
        return set_error(NVBT_EINVAL, "slot %llu: missing continuation slot", (unsigned long long)(i + q));
    if (k >= cap) return set_error(NVBT_EINVAL, "output capacity %llu too small", (unsigned long long)cap);
    decode_group(fmt, s0, ss, o + k * RECORD_BYTES);
    ++k;
    i += g;
  }
  *n_out = k;
  return NVBT_OK;
}

int nvbt_decode_compact(const void* slots, uint64_t n, void* out, uint64_t cap, uint64_t* n_out) {
  return nvbt_decode_slots(slots, n, COMPACT_BYTES, out, cap, n_out);
}

int nvbt_digest_records(const void* records, uint64_t n, nvbt_digest* out) {
  if (!out || (!records && n)) return set_error(NVBT_EINVAL, "null argument");
  out->n_rec = n;
  out->d1 = out->d2 = 0;
  digest_range(static_cast<const unsigned char*>(records), n, &out->d1, &out->d2);
  return NVBT_OK;
}

}  // extern "C"
