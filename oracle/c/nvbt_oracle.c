/* nvbt CPU oracle, multithreaded C edition — TEST INFRASTRUCTURE ONLY.
 *
 * What it is: the same plain, event-by-event application of docs/EVENT_MODEL.md (EM) as the numpy
 * oracle (oracle/events.py + oracle/models/*.py), written a second time in C so that BASELINE.json's
 * full-size configs (C2 1024^3, C3 R-MAT scale 20, C4 8192^2 x 100 with 1.26 G trace records, C5 10^10
 * generated events) can be checked against the GPU element by element. Every workload is walked in
 * program order, one warp and one dynamic instance at a time; every event goes through apply_event(),
 * which is EM §2 written out. Work is split over host threads by warp range (C1-C4) or event-index range
 * (C5); every thread owns its accumulator and the accumulators are summed at the end — all results are
 * sums of non-negative integers (EM §4), so the split cannot change them.
 *
 * Who may use it: only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs (through oracle/coracle.py). It shares no code with the CUDA path
 * (paper_conf_micro_villasnk19_b200/): no header, table or helper of the library is included; program
 * tables arrive as arguments from oracle/programs.py.
 *
 * Pins (tests/test_oracle_c.py, -m "not gpu"): element-by-element equality with the numpy oracle (itself
 * pinned by brute force, the paper's Listing 8 example, published splitmix64 outputs and closed forms) on
 * random event streams and on every workload at small sizes; S/L against Python set definitions on random
 * and adversarial 32-lane events; generator bytes against oracle/gen.py; closed forms (SURVEY I-3) of
 * SGEMM and the stencil at several sizes; partition additivity across thread counts.
 *
 * Citations: P:Lnnn (§x) = /root/reference/PAPER.md line nnn; R-n = DESIGN.md §3 readings.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef uint64_t u64;
typedef uint32_t u32;
typedef int64_t i64;

enum { K_ALU = 0, K_CTRL = 1, K_GLD = 2, K_GST = 3, K_GATOM = 4, K_OTHERMEM = 5 };
#define FULL 0xFFFFFFFFu

/* ------------------------------------------------------------------------------------------------
 * Program table (EM §3): per pc opcode, kind, width, bb, is_leader. Supplied by the caller. */
typedef struct {
  u32 n_pcs, n_ops, n_bbs;
  const int32_t* opcode;
  const int32_t* kind;
  const int32_t* width;
  const int32_t* bb;
  const int32_t* is_leader;
} oprog;

static int is_mem_kind(int k) { return k == K_GLD || k == K_GST || k == K_GATOM; }  /* R-8 */

/* ------------------------------------------------------------------------------------------------
 * Accumulators (EM §2, §4). Flat result layout handed back to Python (int64 words):
 *   counts[4] | H_t[O] | H_w[O] | Ent_t[B] | Ent_w[B] | Ins_t[B] | Ins_w[B] | mem_n[P] | mem_S[P] |
 *   mem_L[P] | hS[33] | hL[33] | trace[3] = (N_rec, D1, D2) | PW_T[W] | PW_W[W]   (W = 0 without per-warp)
 */
typedef struct {
  u64 counts[4];            /* T_issued, T_exec, W_issued, W_exec */
  u64 *H_t, *H_w;           /* [n_ops] */
  u64 *Ent_t, *Ent_w, *Ins_t, *Ins_w;   /* [n_bbs] */
  u64 *mem_n, *mem_S, *mem_L;           /* [n_pcs] */
  u64 hS[33], hL[33];
  u64 n_rec, d1, d2;        /* trace multiset digest (EM §5) */
  u64 *PW_T, *PW_W;         /* [n_warps] or NULL */
  u64 n_warps;
  int trace;
} oacc;

size_t orc_result_words(u32 n_pcs, u32 n_ops, u32 n_bbs, u64 n_warps) {
  return 4 + 2ull * n_ops + 4ull * n_bbs + 3ull * n_pcs + 66 + 3 + 2ull * n_warps;
}

static int acc_init(oacc* a, const oprog* p, u64 n_warps, int trace) {
  memset(a, 0, sizeof *a);
  a->H_t = calloc(2ull * p->n_ops, 8);
  a->Ent_t = calloc(4ull * p->n_bbs, 8);
  a->mem_n = calloc(3ull * p->n_pcs, 8);
  if (!a->H_t || !a->Ent_t || !a->mem_n) return -1;
  a->H_w = a->H_t + p->n_ops;
  a->Ent_w = a->Ent_t + p->n_bbs;
  a->Ins_t = a->Ent_t + 2ull * p->n_bbs;
  a->Ins_w = a->Ent_t + 3ull * p->n_bbs;
  a->mem_S = a->mem_n + p->n_pcs;
  a->mem_L = a->mem_n + 2ull * p->n_pcs;
  a->n_warps = n_warps;
  if (n_warps) {
    a->PW_T = calloc(2ull * n_warps, 8);
    if (!a->PW_T) return -1;
    a->PW_W = a->PW_T + n_warps;
  }
  a->trace = trace;
  return 0;
}

static void acc_free(oacc* a) {
  free(a->H_t);
  free(a->Ent_t);
  free(a->mem_n);
  free(a->PW_T);
}

/* out += a, in the flat layout above */
static void acc_add_to(const oacc* a, const oprog* p, i64* out) {
  u64* o = (u64*)out;
  size_t k = 0;
  for (int i = 0; i < 4; ++i) o[k++] += a->counts[i];
  for (u32 i = 0; i < 2 * p->n_ops; ++i) o[k++] += a->H_t[i];
  for (u32 i = 0; i < 4 * p->n_bbs; ++i) o[k++] += a->Ent_t[i];
  for (u32 i = 0; i < 3 * p->n_pcs; ++i) o[k++] += a->mem_n[i];
  for (int i = 0; i < 33; ++i) o[k++] += a->hS[i];
  for (int i = 0; i < 33; ++i) o[k++] += a->hL[i];
  o[k++] += a->n_rec;
  o[k++] += a->d1;
  o[k++] += a->d2;
  for (u64 i = 0; i < 2 * a->n_warps; ++i) o[k++] += a->PW_T[i];
}

/* ------------------------------------------------------------------------------------------------
 * splitmix64 finaliser and the counter-based generator (EM §3.5; also the digest constants, EM §5). */
static u64 mix64(u64 z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static u64 gen_K(u64 seed, u64 f) { return mix64(seed ^ (f * 0xD1B54A32D192ED03ull)); }

u64 orc_mix64(u64 z) { return mix64(z); }

/* ------------------------------------------------------------------------------------------------
 * EM §2 item 4: S = |{addr[l] >> 5 : l in E}|, L = |{addr[l] >> 7 : l in E}| (Listing 8, P:L189-213,
 * P:L263; R-3: group of equal line addresses; R-5: exact distinct count, which is what the listing's
 * sum of 1/cnt over the lanes equals; R-6: 32 B sectors, 128 B lines). Plain definition: collect the
 * sector keys of the lanes of E, sort them, count the positions where the key changes; lines are
 * sector >> 2, so the same sorted list also orders the line keys. */
static void sectors_lines(const u64* addr, u32 E, u32* S, u32* L) {
  u64 k[32];
  int n = 0;
  for (int l = 0; l < 32; ++l)
    if (E >> l & 1u) k[n++] = addr[l] >> 5;
  for (int i = 1; i < n; ++i) {           /* insertion sort */
    u64 v = k[i];
    int j = i - 1;
    while (j >= 0 && k[j] > v) {
      k[j + 1] = k[j];
      --j;
    }
    k[j + 1] = v;
  }
  u32 s = 0, ln = 0;
  for (int i = 0; i < n; ++i) {
    if (i == 0 || k[i] != k[i - 1]) ++s;
    if (i == 0 || (k[i] >> 2) != (k[i - 1] >> 2)) ++ln;
  }
  *S = s;
  *L = ln;
}

void orc_sectors_lines(const u64* addr, u32 E, u32* S, u32* L) { sectors_lines(addr, E, S, L); }

/* ------------------------------------------------------------------------------------------------
 * EM §5 trace record digest: the 288-byte record as 36 little-endian u64 words x[0..35];
 * h_k = sum_j x[j] * C_k[j] (mod 2^64), C1[j] = mix64(0x1000 + j) | 1, C2[j] = mix64(0x2000 + j) | 1;
 * D_k += mix64(h_k). */
static u64 C1c[36], C2c[36];
static pthread_once_t c_once = PTHREAD_ONCE_INIT;
static void init_consts(void) {
  for (int j = 0; j < 36; ++j) {
    C1c[j] = mix64(0x1000ull + j) | 1ull;
    C2c[j] = mix64(0x2000ull + j) | 1ull;
  }
}

static void trace_record(oacc* a, const oprog* p, u32 launch, u32 warp, u32 seq, u32 pc, u32 A, u32 P,
                         const u64* addr) {
  const u32 E = A & P;
  u64 x[36];
  x[0] = (u64)launch | (u64)warp << 32;
  x[1] = (u64)seq | (u64)pc << 32;
  x[2] = (u64)A | (u64)P << 32;
  x[3] = (u64)(uint16_t)p->opcode[pc] | (u64)(uint8_t)p->width[pc] << 16 | (u64)(uint8_t)p->kind[pc] << 24;
  for (int l = 0; l < 32; ++l) x[4 + l] = (E >> l & 1u) ? addr[l] : 0;   /* R-13: 0 outside E */
  u64 h1 = 0, h2 = 0;
  for (int j = 0; j < 36; ++j) {
    h1 += x[j] * C1c[j];
    h2 += x[j] * C2c[j];
  }
  a->n_rec += 1;
  a->d1 += mix64(h1);
  a->d2 += mix64(h2);
}

/* ------------------------------------------------------------------------------------------------
 * One warp-level event (EM §1-§2). `seq` = records this warp emitted earlier in this launch (EM §5),
 * advanced here. addr may be NULL for non-memory pcs. */
typedef struct {
  u32 launch, warp, seq;
} wctx;

static void apply_event(oacc* a, const oprog* p, wctx* w, u32 pc, u32 A, u32 P, const u64* addr) {
  if (A == 0) return;                              /* EM §1: no event */
  const u32 E = A & P;                             /* R-1: a false guard does not execute */
  const u64 pA = (u64)__builtin_popcount(A), pE = (u64)__builtin_popcount(E), ex = E != 0;
  /* 1. counts: Listing 1 (P:L80-89 (§3)), thread and warp level (R-9, P:L295 (§6.3)) */
  a->counts[0] += pA;
  a->counts[1] += pE;
  a->counts[2] += 1;
  a->counts[3] += ex;
  if (a->PW_T) {
    a->PW_T[w->warp] += pE;
    a->PW_W[w->warp] += ex;
  }
  /* 2. opcode histogram: §6.2 "Top-5 instructions" tool (R-11) */
  const int op = p->opcode[pc];
  a->H_t[op] += pE;
  a->H_w[op] += ex;
  /* 3. basic blocks (P:L89 (§3), BB rule P:L115-117 (§4)): executed instructions per block, and at a
   *    block's first instruction the entries — every active thread enters, whatever its guard */
  const int b = p->bb[pc];
  a->Ins_t[b] += pE;
  a->Ins_w[b] += ex;
  if (p->is_leader[pc]) {
    a->Ent_t[b] += pA;
    a->Ent_w[b] += 1;
  }
  /* 4. memory divergence + 5. trace record: global LD/ST/ATOM events that execute (R-8, R-10) */
  if (is_mem_kind(p->kind[pc]) && E != 0) {
    u32 S, L;
    sectors_lines(addr, E, &S, &L);
    a->mem_n[pc] += 1;
    a->mem_S[pc] += S;
    a->mem_L[pc] += L;
    a->hS[S] += 1;
    a->hL[L] += 1;
    if (a->trace) trace_record(a, p, w->launch, w->warp, w->seq, pc, A, P, addr);
    w->seq += 1;
  }
}

/* mask with bit l set where c[l] != 0 */
static u32 mask_of(const int* c) {
  u32 m = 0;
  for (int l = 0; l < 32; ++l)
    if (c[l]) m |= 1u << l;
  return m;
}

/* ------------------------------------------------------------------------------------------------
 * Thread pool plumbing: run fn(job, lo, hi, acc) for T contiguous shares of [0, n), one accumulator per
 * thread, then sum the accumulators into out. */
typedef struct job_s job_t;
typedef void (*range_fn)(const job_t* job, u64 lo, u64 hi, oacc* acc);
struct job_s {
  const oprog* prog;
  range_fn fn;
  u64 n_warps_pw;   /* per-warp array length (0 = none) */
  int trace;
  /* workload parameters */
  i64 M, N, K, n, iters;
  u64 p0, p1, p2, p3, p4, p5, p6;
  u32 launch;
  u64 seed, first;
  const int32_t* rowptr;
  const int32_t* col;
  const uint8_t *mask, *visited, *updating;   /* BFS state at the launch's start */
  int kernel;                                   /* BFS kernel 1 or 2 */
  /* event-list input (orc_events) */
  const u32 *ev_warp, *ev_pc, *ev_A, *ev_P;
  const u64* ev_addr;
};

typedef struct {
  const job_t* job;
  u64 lo, hi;
  oacc acc;
  int rc;
} part_t;

static void* part_main(void* arg) {
  part_t* t = (part_t*)arg;
  t->job->fn(t->job, t->lo, t->hi, &t->acc);
  return NULL;
}

static int run_parallel(const job_t* job, u64 lo, u64 hi, int threads, i64* out) {
  pthread_once(&c_once, init_consts);
  if (threads < 1) threads = 1;
  u64 n = hi - lo;
  if ((u64)threads > n && n > 0) threads = (int)n;
  part_t* parts = calloc((size_t)threads, sizeof(part_t));
  pthread_t* tids = calloc((size_t)threads, sizeof(pthread_t));
  if (!parts || !tids) return -1;
  int rc = 0;
  for (int t = 0; t < threads; ++t) {
    parts[t].job = job;
    parts[t].lo = lo + n * (u64)t / (u64)threads;
    parts[t].hi = lo + n * (u64)(t + 1) / (u64)threads;
    if (acc_init(&parts[t].acc, job->prog, job->n_warps_pw, job->trace)) rc = -1;
  }
  if (rc == 0) {
    for (int t = 1; t < threads; ++t) pthread_create(&tids[t], NULL, part_main, &parts[t]);
    part_main(&parts[0]);
    for (int t = 1; t < threads; ++t) pthread_join(tids[t], NULL);
    for (int t = 0; t < threads; ++t) acc_add_to(&parts[t].acc, job->prog, out);
  }
  for (int t = 0; t < threads; ++t) acc_free(&parts[t].acc);
  free(parts);
  free(tids);
  return rc;
}

/* ------------------------------------------------------------------------------------------------
 * Arbitrary event lists (the numpy Accumulator.add interface): event i = (warp[i], pc[i], A[i], P[i],
 * addr[32 i .. 32 i + 31]); all events belong to launch `launch`; a warp's records are numbered in list
 * order. Single-threaded (seq depends on the order). */
static void events_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  /* seq per warp: small lists only, linear scan of earlier events of the same warp */
  for (u64 i = lo; i < hi; ++i) {
    wctx w = {j->launch, j->ev_warp[i], 0};
    for (u64 k = 0; k < i; ++k)
      if (j->ev_warp[k] == w.warp && is_mem_kind(j->prog->kind[j->ev_pc[k]]) && (j->ev_A[k] & j->ev_P[k]) != 0) w.seq++;
    apply_event(a, j->prog, &w, j->ev_pc[i], j->ev_A[i], j->ev_P[i], j->ev_addr ? j->ev_addr + 32 * i : NULL);
  }
}

int orc_events(const oprog* p, u32 launch, u64 n, const u32* warp, const u32* pc, const u32* A, const u32* P,
               const u64* addr, u64 n_warps_pw, int trace, i64* out) {
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p;
  j.fn = events_range;
  j.n_warps_pw = n_warps_pw;
  j.trace = trace;
  j.launch = launch;
  j.ev_warp = warp;
  j.ev_pc = pc;
  j.ev_A = A;
  j.ev_P = P;
  j.ev_addr = addr;
  for (u64 i = 0; i < n; ++i) {
    if (pc[i] >= p->n_pcs) return -2;
    if (n_warps_pw && warp[i] >= n_warps_pw) return -2;
    if (is_mem_kind(p->kind[pc[i]]) && (A[i] & P[i]) && !addr) return -2;
  }
  return run_parallel(&j, 0, n, 1, out);
}

/* ------------------------------------------------------------------------------------------------
 * C1 vectorAdd, EM §3.1: c[i] = a[i] + b[i], i = ctaid.x*256 + tid.x = 32 w + l (CTA 256 = 8 warps).
 * pcs 0-3 every lane; pc 4 `@P0 EXIT`, P0 = (i >= N), issued by all lanes; lanes that executed EXIT are
 * gone for pcs 5-12. Buffers: p0 = a, p1 = b, p2 = c. */
static void vectoradd_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  const oprog* p = j->prog;
  for (u64 w = lo; w < hi; ++w) {
    wctx wc = {j->launch, (u32)w, 0};
    int ge[32], lt[32];
    u64 ad[32], bd[32], cd[32];
    for (int l = 0; l < 32; ++l) {
      const i64 i = 32 * (i64)w + l;
      ge[l] = i >= j->N;
      lt[l] = !ge[l];
      ad[l] = j->p0 + 4 * (u64)i;
      bd[l] = j->p1 + 4 * (u64)i;
      cd[l] = j->p2 + 4 * (u64)i;
    }
    for (u32 pc = 0; pc < 4; ++pc) apply_event(a, p, &wc, pc, FULL, FULL, NULL);
    apply_event(a, p, &wc, 4, FULL, mask_of(ge), NULL);            /* @P0 EXIT */
    const u32 A = mask_of(lt);
    for (u32 pc = 5; pc <= 12; ++pc)
      apply_event(a, p, &wc, pc, A, A, pc == 7 ? ad : pc == 8 ? bd : pc == 11 ? cd : NULL);
  }
}

int orc_vectoradd(const oprog* p, i64 N, u64 a, u64 b, u64 c, u32 launch, u64 w0, u64 w1, int threads,
                  u64 n_warps_pw, int trace, i64* out) {
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p; j.fn = vectoradd_range; j.n_warps_pw = n_warps_pw; j.trace = trace;
  j.N = N; j.p0 = a; j.p1 = b; j.p2 = c; j.launch = launch;
  return run_parallel(&j, w0, w1, threads, out);
}

/* ------------------------------------------------------------------------------------------------
 * C2 naive SGEMM, EM §3.2: CTA (32, 8), grid (gx, gy) = (ceil(M/32), ceil(N/8)); warp w: linear CTA
 * w / 8 = ctaid.x + ctaid.y gx, tid.y = w % 8; lane l: row = ctaid.x*32 + l, col = ctaid.y*8 + tid.y.
 * Buffers p0 = A (M x K), p1 = B (K x N), p2 = C (M x N), fp32 row-major. */
static void sgemm_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  const oprog* p = j->prog;
  const i64 M = j->M, N = j->N, K = j->K, gx = (M + 31) / 32;
  for (u64 w = lo; w < hi; ++w) {
    wctx wc = {j->launch, (u32)w, 0};
    const i64 cta = (i64)w / 8, ty = (i64)w % 8;
    const i64 cx = cta % gx, cy = cta / gx;
    const i64 col = cy * 8 + ty;
    i64 row[32];
    int p0[32], live[32];
    for (int l = 0; l < 32; ++l) {
      row[l] = cx * 32 + l;
      p0[l] = row[l] >= M || col >= N;
      live[l] = !p0[l];
    }
    for (u32 pc = 0; pc <= 6; ++pc) apply_event(a, p, &wc, pc, FULL, FULL, NULL);  /* S2R x4, IMAD x2, ISETP */
    apply_event(a, p, &wc, 7, FULL, mask_of(p0), NULL);                            /* @P0 EXIT */
    const u32 A = mask_of(live);
    apply_event(a, p, &wc, 8, A, A, NULL);                                         /* MOV acc */
    apply_event(a, p, &wc, 9, A, A, NULL);                                         /* MOV k */
    u64 ad[32], bd[32];
    for (i64 k = 0; k < K; ++k) {                                                  /* BB2 instance k */
      for (int l = 0; l < 32; ++l) {
        ad[l] = j->p0 + 4 * (u64)(row[l] * K + k);
        bd[l] = j->p1 + 4 * (u64)(k * N + col);
      }
      apply_event(a, p, &wc, 10, A, A, ad);                                        /* LDG A[row][k] */
      apply_event(a, p, &wc, 11, A, A, bd);                                        /* LDG B[k][col] */
      apply_event(a, p, &wc, 12, A, A, NULL);                                      /* FFMA */
      apply_event(a, p, &wc, 13, A, A, NULL);                                      /* IADD */
      apply_event(a, p, &wc, 14, A, A, NULL);                                      /* ISETP */
      apply_event(a, p, &wc, 15, A, k + 1 < K ? A : 0u, NULL);                     /* @P1 BRA, P1 = k+1 < K */
    }
    for (int l = 0; l < 32; ++l) ad[l] = j->p2 + 4 * (u64)(row[l] * N + col);
    apply_event(a, p, &wc, 16, A, A, ad);                                          /* STG C[row][col] */
    apply_event(a, p, &wc, 17, A, A, NULL);                                        /* EXIT */
  }
}

int orc_sgemm(const oprog* p, i64 M, i64 N, i64 K, u64 A, u64 B, u64 C, u32 launch, u64 w0, u64 w1,
              int threads, u64 n_warps_pw, int trace, i64* out) {
  if (K < 1) return -2;
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p; j.fn = sgemm_range; j.n_warps_pw = n_warps_pw; j.trace = trace;
  j.M = M; j.N = N; j.K = K; j.p0 = A; j.p1 = B; j.p2 = C; j.launch = launch;
  return run_parallel(&j, w0, w1, threads, out);
}

/* ------------------------------------------------------------------------------------------------
 * C4 5-point Jacobi stencil, EM §3.4: CTA (32, 8), grid (ceil(n/32), ceil(n/8)); lane l of warp w:
 * j = ctaid.x*32 + l (column), i = ctaid.y*8 + tid.y (row); P1 = 0 < i < n-1 and 0 < j < n-1.
 * Iteration it (launch first_launch + it) reads buffer it % 2 and writes (it + 1) % 2 (p0 = buffer 0,
 * p1 = buffer 1). Warps [lo, hi) of every iteration. */
static void stencil_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  const oprog* p = j->prog;
  const i64 n = j->n, gx = (n + 31) / 32;
  for (i64 it = 0; it < j->iters; ++it) {
    const u64 in = (it % 2) ? j->p1 : j->p0, out = (it % 2) ? j->p0 : j->p1;
    for (u64 w = lo; w < hi; ++w) {
      wctx wc = {j->launch + (u32)it, (u32)w, 0};
      const i64 cta = (i64)w / 8, ty = (i64)w % 8;
      const i64 i = (cta / gx) * 8 + ty;
      int p0[32], live[32], p1[32];
      i64 jj[32];
      for (int l = 0; l < 32; ++l) {
        jj[l] = (cta % gx) * 32 + l;
        p0[l] = i >= n || jj[l] >= n;
        live[l] = !p0[l];
        p1[l] = live[l] && i > 0 && i < n - 1 && jj[l] > 0 && jj[l] < n - 1;
      }
      for (u32 pc = 0; pc <= 6; ++pc) apply_event(a, p, &wc, pc, FULL, FULL, NULL);
      apply_event(a, p, &wc, 7, FULL, mask_of(p0), NULL);                           /* @P0 EXIT */
      const u32 A = mask_of(live), P1 = mask_of(p1);
      u64 ad[32];
      apply_event(a, p, &wc, 8, A, A, NULL);                                        /* ISETP P1 */
      for (int l = 0; l < 32; ++l) ad[l] = in + 4 * (u64)(i * n + jj[l]);
      apply_event(a, p, &wc, 9, A, A, ad);                                          /* center */
      for (int l = 0; l < 32; ++l) ad[l] = in + 4 * (u64)((i - 1) * n + jj[l]);
      apply_event(a, p, &wc, 10, A, P1, ad);                                        /* @P1 up */
      for (int l = 0; l < 32; ++l) ad[l] = in + 4 * (u64)((i + 1) * n + jj[l]);
      apply_event(a, p, &wc, 11, A, P1, ad);                                        /* @P1 down */
      for (int l = 0; l < 32; ++l) ad[l] = in + 4 * (u64)(i * n + jj[l] - 1);
      apply_event(a, p, &wc, 12, A, P1, ad);                                        /* @P1 left */
      for (int l = 0; l < 32; ++l) ad[l] = in + 4 * (u64)(i * n + jj[l] + 1);
      apply_event(a, p, &wc, 13, A, P1, ad);                                        /* @P1 right */
      for (u32 pc = 14; pc <= 17; ++pc) apply_event(a, p, &wc, pc, A, P1, NULL);    /* @P1 FADD x3, FMUL */
      apply_event(a, p, &wc, 18, A, A, NULL);                                       /* SEL */
      for (int l = 0; l < 32; ++l) ad[l] = out + 4 * (u64)(i * n + jj[l]);
      apply_event(a, p, &wc, 19, A, A, ad);                                         /* STG out */
      apply_event(a, p, &wc, 20, A, A, NULL);                                       /* EXIT */
    }
  }
}

int orc_stencil(const oprog* p, i64 n, u64 buf0, u64 buf1, i64 iters, u32 first_launch, u64 w0, u64 w1,
                int threads, int trace, i64* out) {
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p; j.fn = stencil_range; j.trace = trace;
  j.n = n; j.iters = iters; j.p0 = buf0; j.p1 = buf1; j.launch = first_launch;
  return run_parallel(&j, w0, w1, threads, out);
}

/* ------------------------------------------------------------------------------------------------
 * C3 BFS, EM §3.3 (two kernels, one pc namespace; CTA 256, t = 32 w + l). Buffers: p0 mask, p1 visited,
 * p2 updating, p3 cost, p4 over, p5 rowptr, p6 col (device byte addresses, only used to form event
 * addresses). The events of a launch depend only on the state at its start (kernel 1 reads mask,
 * visited, rowptr, col; kernel 2 reads updating), which the job carries. */
static void bfs1_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  const oprog* p = j->prog;
  const i64 n = j->n;
  for (u64 w = lo; w < hi; ++w) {
    wctx wc = {j->launch, (u32)w, 0};
    i64 t[32], start[32], end[32], deg[32];
    int live[32], fr[32], dead[32], nofr[32], empty[32];
    u64 ad[32];
    for (int l = 0; l < 32; ++l) {
      t[l] = 32 * (i64)w + l;
      live[l] = t[l] < n;
      dead[l] = !live[l];
    }
    for (u32 pc = 0; pc < 4; ++pc) apply_event(a, p, &wc, pc, FULL, FULL, NULL);
    apply_event(a, p, &wc, 4, FULL, mask_of(dead), NULL);                     /* @P0 EXIT, P0 = t >= n */
    const u32 Alive = mask_of(live);
    for (int l = 0; l < 32; ++l) ad[l] = j->p0 + (u64)t[l];
    apply_event(a, p, &wc, 5, Alive, Alive, ad);                              /* LDG mask[t] */
    apply_event(a, p, &wc, 6, Alive, Alive, NULL);                            /* ISETP */
    for (int l = 0; l < 32; ++l) {
      fr[l] = live[l] && j->mask[t[l]] != 0;
      nofr[l] = live[l] && !fr[l];
    }
    apply_event(a, p, &wc, 7, Alive, mask_of(nofr), NULL);                    /* @!P1 BRA */
    const u32 Af = mask_of(fr);
    i64 maxdeg = 0;
    for (int l = 0; l < 32; ++l) {
      start[l] = fr[l] ? j->rowptr[t[l]] : 0;
      end[l] = fr[l] ? j->rowptr[t[l] + 1] : 0;
      deg[l] = end[l] - start[l];
      empty[l] = fr[l] && start[l] >= end[l];
      if (deg[l] > maxdeg) maxdeg = deg[l];
    }
    for (int l = 0; l < 32; ++l) ad[l] = j->p0 + (u64)t[l];
    apply_event(a, p, &wc, 8, Af, Af, ad);                                    /* STG mask[t] = 0 */
    for (int l = 0; l < 32; ++l) ad[l] = j->p5 + 4 * (u64)t[l];
    apply_event(a, p, &wc, 9, Af, Af, ad);                                    /* LDG rowptr[t] */
    for (int l = 0; l < 32; ++l) ad[l] = j->p5 + 4 * (u64)(t[l] + 1);
    apply_event(a, p, &wc, 10, Af, Af, ad);                                   /* LDG rowptr[t+1] */
    apply_event(a, p, &wc, 11, Af, Af, NULL);                                 /* ISETP */
    apply_event(a, p, &wc, 12, Af, mask_of(empty), NULL);                     /* @P2 BRA, P2 = start >= end */
    for (i64 k = 0; k < maxdeg; ++k) {                                        /* edge-loop instance k */
      int ak[32], vis[32], unv[32], more[32];
      i64 e[32], nb[32];
      for (int l = 0; l < 32; ++l) {
        ak[l] = deg[l] > k;
        e[l] = ak[l] ? start[l] + k : 0;
        nb[l] = ak[l] ? j->col[e[l]] : 0;
        vis[l] = ak[l] && j->visited[nb[l]] != 0;
        unv[l] = ak[l] && !vis[l];
        more[l] = ak[l] && e[l] + 1 < end[l];
      }
      const u32 Ak = mask_of(ak);
      for (int l = 0; l < 32; ++l) ad[l] = j->p6 + 4 * (u64)e[l];
      apply_event(a, p, &wc, 13, Ak, Ak, ad);                                 /* LDG col[e] */
      for (int l = 0; l < 32; ++l) ad[l] = j->p1 + (u64)nb[l];
      apply_event(a, p, &wc, 14, Ak, Ak, ad);                                 /* LDG visited[col[e]] */
      apply_event(a, p, &wc, 15, Ak, Ak, NULL);                               /* ISETP */
      apply_event(a, p, &wc, 16, Ak, mask_of(vis), NULL);                     /* @P3 BRA, P3 = visited */
      const u32 Au = mask_of(unv);
      for (int l = 0; l < 32; ++l) ad[l] = j->p2 + (u64)nb[l];
      apply_event(a, p, &wc, 17, Au, Au, ad);                                 /* STG updating[col[e]] = 1 */
      apply_event(a, p, &wc, 18, Ak, Ak, NULL);                               /* IADD */
      apply_event(a, p, &wc, 19, Ak, Ak, NULL);                               /* ISETP */
      apply_event(a, p, &wc, 20, Ak, mask_of(more), NULL);                    /* @P4 BRA, P4 = e+1 < end */
    }
    apply_event(a, p, &wc, 21, Alive, Alive, NULL);                           /* EXIT */
  }
}

static void bfs2_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  const oprog* p = j->prog;
  const i64 n = j->n;
  for (u64 w = lo; w < hi; ++w) {
    wctx wc = {j->launch, (u32)w, 0};
    i64 t[32];
    int live[32], dead[32], u[32], nu[32];
    u64 ad[32];
    for (int l = 0; l < 32; ++l) {
      t[l] = 32 * (i64)w + l;
      live[l] = t[l] < n;
      dead[l] = !live[l];
    }
    for (u32 pc = 22; pc < 26; ++pc) apply_event(a, p, &wc, pc, FULL, FULL, NULL);
    apply_event(a, p, &wc, 26, FULL, mask_of(dead), NULL);                    /* @P0 EXIT */
    const u32 Alive = mask_of(live);
    for (int l = 0; l < 32; ++l) ad[l] = j->p2 + (u64)t[l];
    apply_event(a, p, &wc, 27, Alive, Alive, ad);                             /* LDG updating[t] */
    apply_event(a, p, &wc, 28, Alive, Alive, NULL);
    for (int l = 0; l < 32; ++l) {
      u[l] = live[l] && j->updating[t[l]] != 0;
      nu[l] = live[l] && !u[l];
    }
    apply_event(a, p, &wc, 29, Alive, mask_of(nu), NULL);                     /* @!P1 BRA */
    const u32 Au = mask_of(u);
    for (int l = 0; l < 32; ++l) ad[l] = j->p0 + (u64)t[l];
    apply_event(a, p, &wc, 30, Au, Au, ad);                                   /* STG mask = 1 */
    for (int l = 0; l < 32; ++l) ad[l] = j->p1 + (u64)t[l];
    apply_event(a, p, &wc, 31, Au, Au, ad);                                   /* STG visited = 1 */
    for (int l = 0; l < 32; ++l) ad[l] = j->p3 + 4 * (u64)t[l];
    apply_event(a, p, &wc, 32, Au, Au, ad);                                   /* STG cost = level + 1 */
    for (int l = 0; l < 32; ++l) ad[l] = j->p2 + (u64)t[l];
    apply_event(a, p, &wc, 33, Au, Au, ad);                                   /* STG updating = 0 */
    for (int l = 0; l < 32; ++l) ad[l] = j->p4;
    apply_event(a, p, &wc, 34, Au, Au, ad);                                   /* STG over = 1 */
    apply_event(a, p, &wc, 35, Alive, Alive, NULL);                           /* EXIT */
  }
}

/* Whole BFS from src (EM §3.3 host loop): level = 0; do { over = 0; updating[:] = 0; K1; K2(level);
 * level += 1 } while (over). Launch ids first_launch, first_launch + 1, ... (K1 and K2 alternate).
 * Instrumented warps [w0, w1) of every launch; the state is always simulated for every vertex.
 * ptrs[7] = mask, visited, updating, cost, over, rowptr, col. cost_out[n] (nullable), *levels_out. */
int orc_bfs(const oprog* p, i64 n, const int32_t* rowptr, const int32_t* col, i64 src, const u64* ptrs,
            u32 first_launch, u64 w0, u64 w1, int threads, u64 n_warps_pw, int trace, i64* out,
            int32_t* cost_out, i64* levels_out) {
  uint8_t* mask = calloc((size_t)n, 1);
  uint8_t* visited = calloc((size_t)n, 1);
  uint8_t* updating = calloc((size_t)n, 1);
  int32_t* cost = malloc(4 * (size_t)n);
  if (!mask || !visited || !updating || !cost) return -1;
  for (i64 v = 0; v < n; ++v) cost[v] = -1;
  mask[src] = visited[src] = 1;
  cost[src] = 0;
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p; j.n_warps_pw = n_warps_pw; j.trace = trace; j.n = n;
  j.p0 = ptrs[0]; j.p1 = ptrs[1]; j.p2 = ptrs[2]; j.p3 = ptrs[3]; j.p4 = ptrs[4]; j.p5 = ptrs[5]; j.p6 = ptrs[6];
  j.rowptr = rowptr; j.col = col;
  j.mask = mask; j.visited = visited; j.updating = updating;
  i64 level = 0;
  u32 launch = first_launch;
  int rc = 0;
  for (;;) {
    memset(updating, 0, (size_t)n);
    /* kernel 1 (expand): events, then its state change — frontier masks cleared, unvisited neighbours
     * of frontier vertices marked in updating */
    j.fn = bfs1_range; j.launch = launch++;
    if ((rc = run_parallel(&j, w0, w1, threads, out))) break;
    for (i64 v = 0; v < n; ++v) {
      if (!mask[v]) continue;
      mask[v] = 0;
      for (i64 e = rowptr[v]; e < rowptr[v + 1]; ++e)
        if (!visited[col[e]]) updating[col[e]] = 1;
    }
    /* kernel 2 (update, level): events, then every vertex with updating set joins the frontier */
    j.fn = bfs2_range; j.launch = launch++;
    if ((rc = run_parallel(&j, w0, w1, threads, out))) break;
    int over = 0;
    for (i64 v = 0; v < n; ++v) {
      if (!updating[v]) continue;
      mask[v] = visited[v] = 1;
      cost[v] = (int32_t)(level + 1);
      updating[v] = 0;
      over = 1;
    }
    level += 1;
    if (!over) break;
  }
  if (cost_out) memcpy(cost_out, cost, 4 * (size_t)n);
  if (levels_out) *levels_out = level;
  free(mask); free(visited); free(updating); free(cost);
  return rc;
}

/* ------------------------------------------------------------------------------------------------
 * C5 generator (EM §3.5), event i for seed `seed`:
 *   pc = R(i,0) % 4096; warp = R(i,1) % 2^20
 *   A = (R(i,2) % 4 != 0) ? 0xFFFFFFFF : low32(R(i,3)); if A == 0: A = 1
 *   P = (R(i,4) % 8 < 6) ? 0xFFFFFFFF : low32(R(i,5))
 *   memory pc: wd = width(pc); pat = R(i,6) % 6; base = (R(i,7) & (2^40-1)) & ~127; s = R(i,8);
 *     lane l, r = R(i, 64 + l): pat 0 base + l wd | 1 base + l (wd << (s % 10)) | 2 base |
 *     3 base + (r % (4096/wd)) wd | 4 (r & (2^40-1)) & ~(wd-1) | 5 base + (l ^ (s & 31)) wd
 * with R(i, f) = mix64(K(f) ^ i), K(f) = mix64(seed ^ f * 0xD1B54A32D192ED03). */
typedef struct {
  u64 k[96];
} gkeys;

static void gen_keys(gkeys* g, u64 seed) {
  for (int f = 0; f < 96; ++f) g->k[f] = gen_K(seed, (u64)f);
}

static void gen_event(const gkeys* g, const oprog* p, u64 i, u32* pc, u32* warp, u32* A, u32* P, u64* addr) {
#define R(f) mix64(g->k[f] ^ i)
  *pc = (u32)(R(0) % 4096);
  *warp = (u32)(R(1) % (1ull << 20));
  *A = (R(2) % 4 != 0) ? FULL : (u32)R(3);
  if (*A == 0) *A = 1;
  *P = (R(4) % 8 < 6) ? FULL : (u32)R(5);
  if (addr && is_mem_kind(p->kind[*pc])) {
    const u64 wd = (u64)p->width[*pc], pat = R(6) % 6;
    const u64 base = (R(7) & ((1ull << 40) - 1)) & ~127ull, s = R(8);
    for (u64 l = 0; l < 32; ++l) {
      switch (pat) {
        case 0: addr[l] = base + l * wd; break;
        case 1: addr[l] = base + l * (wd << (s % 10)); break;
        case 2: addr[l] = base; break;
        case 3: addr[l] = base + (R(64 + l) % (4096 / wd)) * wd; break;
        case 4: addr[l] = (R(64 + l) & ((1ull << 40) - 1)) & ~(wd - 1); break;
        default: addr[l] = base + (l ^ (s & 31)) * wd; break;
      }
    }
  }
#undef R
}

/* Events [first, first + n) as the replay stream layout (EM §3.5): 16 B headers {pc, warp, A, P} at
 * hdr + 16 i and, for memory pcs, 32 x u64 addresses at addr + 256 i (other slots untouched). */
void orc_gen_events(const oprog* p, u64 seed, u64 first, u64 n, u32* hdr, u64* addr) {
  gkeys g;
  gen_keys(&g, seed);
  for (u64 i = 0; i < n; ++i)
    gen_event(&g, p, first + i, hdr + 4 * i, hdr + 4 * i + 1, hdr + 4 * i + 2, hdr + 4 * i + 3, addr + 32 * i);
}

static void replay_range(const job_t* j, u64 lo, u64 hi, oacc* a) {
  gkeys g;
  gen_keys(&g, j->seed);
  u64 ad[32];
  for (u64 i = lo; i < hi; ++i) {
    u32 pc, warp, A, P;
    gen_event(&g, j->prog, i, &pc, &warp, &A, &P, ad);
    wctx wc = {0, warp, 0};
    apply_event(a, j->prog, &wc, pc, A, P, ad);   /* EM §3.5: replay applies §2 items 1-4 */
  }
}

int orc_replay(const oprog* p, u64 seed, u64 first, u64 n, int threads, i64* out) {
  job_t j;
  memset(&j, 0, sizeof j);
  j.prog = p; j.fn = replay_range; j.seed = seed;
  return run_parallel(&j, first, first + n, threads, out);
}
