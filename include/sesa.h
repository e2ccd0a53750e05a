/*
 * sesa.h — C ABI of the B200-native concrete race checker (SESA hot path).
 *
 * Paper: P. Li, G. Li, G. Gopalakrishnan, "Practical Symbolic Race Checking of GPU Programs", SC'14.
 * Citations "P:<line>" refer to /root/reference/PAPER.md (the paper's extracted text) and name the
 * section they fall in.  The paper checks races symbolically, instantiating a barrier interval's read
 * and write sets at two thread ids t1 != t2 (§II; §IV-B).  This library decides the
 * same question exhaustively on CONCRETE access records ("race state" entries `cond ? r|w(addr)` of one
 * thread in one barrier interval, §IV-A), every thread of the real launch geometry at once.
 *
 * Race definition implemented (README of the method, DESIGN.md §2 "readings"):
 *   two access records r != s race at location λ iff
 *     (1) they come from different threads: (block,thread) differ            P:79 (t1 != t2)
 *     (2) at least one is a write (plain WRITE or ATOMIC)                     P:43 (§I definition)
 *     (3) they are not both ATOMIC                                            P:573, P:447 (§VI)
 *     (4) they are unordered: shared memory: same block and same interval
 *         (λ fixes both); global: different blocks, or same block and same
 *         interval                                                            P:73, P:79, P:97 (§II)
 *     (5) lockstep mode only: not (same block, same interval, same warp, one
 *         of them a READ)                                                     P:281 (§IV-B warp execution)
 *     (6) not (both plain WRITE with equal value_hash)  — benign W/W          P:467 Table IV
 *   λ = (SHARED, block, interval, granule) or (GLOBAL, granule); granule = addr / granularity;
 *   a record of `size` bytes covers granules [addr/G, (addr+size-1)/G].     P:43 "same memory location",
 *                                                                            P:269 "address overlapping"
 *   kind = RW if one of them is a READ, else WW (W/W or W/A).              P:79 (WW / WR checks)
 *   One race record per (λ, kind), witnessed by the lexicographically smallest (first, second) pair of
 *   record indices (first < second).  The paper's witnesses are "a solution" of the solver; this
 *   library fixes the canonical one so that results are reproducible (reading R12).
 *   Output order: (epoch, space, block, interval, addr, kind), SHARED < GLOBAL; a global race has
 *   block = interval = 0xFFFFFFFF.
 *
 * Conventions
 *   - Every function returns sesa_status (0 == SESA_OK) unless stated.  Thread-compatible: one handle per
 *     host thread; distinct handles may be used concurrently.
 *   - All-or-nothing: on any error the handle's previous race list is dropped and sesa_races_get returns
 *     SESA_ESTATE until the next successful check.  sesa_last_error() gives a one-line detail.
 *   - Device pointers are plain CUDA device pointers (e.g. torch.Tensor.data_ptr()); streams are
 *     cudaStream_t passed as void* (NULL = legacy default stream).
 */
#ifndef SESA_H
#define SESA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SESA_ABI_VERSION 1

typedef enum {
  SESA_OK = 0,
  SESA_EINVAL = 1, /* bad argument, bad config, or bad record (sesa_last_error names the lowest bad index) */
  SESA_ERANGE = 2, /* a field range does not fit the packed 64-bit sort key, or n / entries >= 2^31      */
  SESA_ENOMEM = 3, /* device or host allocation failed                                                   */
  SESA_ECUDA = 4,  /* a CUDA runtime error; sesa_last_error carries cudaGetErrorString                     */
  SESA_ENCCL = 5,  /* an NCCL error (distributed handles)                                                */
  SESA_ESTATE = 6, /* call not valid in the handle's current state (e.g. races_get with no result)      */
  SESA_ETRUNC = 7  /* sesa_races_get: cap < number of races; cap records copied, *n_races = total       */
} sesa_status;

/* memory spaces (Fig. 3 memory sorts τl / τg; shared vs global) */
enum { SESA_SPACE_SHARED = 0, SESA_SPACE_GLOBAL = 1 };
/* access kinds: load -> READ, store -> WRITE (Fig. 3); any atomic RMW intrinsic -> ATOMIC */
enum { SESA_READ = 0, SESA_WRITE = 1, SESA_ATOMIC = 2 };
/* race kinds ("WW (Write-Write)" and "WR" checks).  SESA_RACE_WW_BENIGN is reported only with
 * SESA_FLAG_REPORT_BENIGN (Table IV "W/W (Benign)" verdicts; "races later deemed to
 * be benign"): a location holding a benign pair = two plain WRITEs with equal value_hash that satisfy
 * rules (1) and (4) above (rules (2), (3) hold for two plain writes; (5) exempts only pairs with a READ).  One
 * record per such location, witnessed by the lexicographically smallest benign pair; rule (6) still keeps
 * these pairs out of SESA_RACE_WW, so a location may carry both a WW and a WW_BENIGN record. */
enum { SESA_RACE_RW = 1, SESA_RACE_WW = 2, SESA_RACE_WW_BENIGN = 3 };
/* sesa_config.flags bits */
enum { SESA_FLAG_REPORT_BENIGN = 1 };

typedef struct {
  uint32_t warp_size;   /* >= 1.  32 = CUDA warp ("groups of 32 consecutively numbered threads");
                           1 = no warp semantics.  warp(r) = r.thread / warp_size              */
  uint32_t lockstep;    /* 0 | 1.  1 = exempt intra-warp pairs with a READ (R6-R8)    */
  uint32_t granularity; /* power of two in [1, 4096]: bytes per comparison unit; 1 = exact byte overlap */
  uint32_t flags;       /* SESA_FLAG_* bits; others must be 0.  SESA_FLAG_REPORT_BENIGN: also report benign
                           W/W locations (kind SESA_RACE_WW_BENIGN), on single-GPU and distributed handles  */
} sesa_config;

/* One concrete access: the paper's race-state entry `c ? r|w(a)` of one thread.
 * 32 bytes, 8-byte aligned, array-of-structs in device memory. */
typedef struct {
  uint64_t addr;       /* SHARED: byte offset in the block's shared window; GLOBAL: device byte address    */
  uint64_t value_hash; /* WRITE: 64-bit hash of the bytes written (producers fold size/offset in if writes
                          of different sizes overlap); ignored for READ/ATOMIC                           */
  uint32_t block;      /* linear blockIdx (x + y*gdx + z*gdx*gdy)                                    */
  uint32_t thread;     /* linear threadIdx (x + y*bdx + z*bdx*bdy)                                   */
  uint32_t interval;   /* number of __syncthreads the block executed before the access ("the code
                          from the beginning to the barrier constitutes the first barrier interval" = 0) */
  uint16_t size;       /* bytes accessed, >= 1                                                             */
  uint8_t space;       /* SESA_SPACE_*                                                                     */
  uint8_t rw;          /* SESA_READ / SESA_WRITE / SESA_ATOMIC                                             */
} sesa_access;

/* One race: one per (location, kind).  40 bytes. */
typedef struct {
  uint64_t addr;            /* granule base address = granule * granularity                              */
  uint64_t first, second;   /* witness record indices (index_base-adjusted), first < second; lexicographic
                               minimum over all racing pairs at this (location, kind)                      */
  uint32_t block, interval; /* SHARED: the location's block and interval; GLOBAL: 0xFFFFFFFF, 0xFFFFFFFF  */
  uint8_t space, kind;      /* SESA_SPACE_*, SESA_RACE_*                                                   */
  uint8_t reserved[2];      /* zero                                                                        */
  uint32_t epoch;           /* the kernel launch of the location (sesa_race_check_launches); else 0        */
} sesa_race;

/* Parametric access descriptor: one access of one parametric flow (§IV).  The paper instantiates
 * a flow's race history at two symbolic thread ids; sesa_expand instantiates it at EVERY thread id of every
 * block of the flow ("replacing every occurrence of i with j").
 *   active(t)  = (t & pmask) == pval  &&  (pmod == 0 || t % pmod == prem)  &&  plo <= t < phi  && t < nthreads
 *                (conditional access `c(i) ? access`; flow condition)
 *   f(t)       = t | (t + fc) % fm | t ^ fc | t >> fc | (t >> fc) * fm + (t & (2^fc - 1))
 *                (fkind = SESA_F_ID / MODADD / XOR / SHR / ROW2D; ROW2D maps a linear tid onto a row-major
 *                 2-D tile: ty = t >> fc, tx = t & (2^fc - 1), f = ty * fm + tx)
 *   invalid: fkind > 4, MODADD with fm == 0, SHR/ROW2D with fc >= 32  -> SESA_EINVAL
 *   addr       = base + bstride*block + tstride*f(t) + istride*k      (mod 2^64, signed strides), k < count
 *   value_hash = rw != SESA_WRITE ? 0 : (flags & SESA_FLOW_CONST_VALUE) ? value_seed
 *                : sesa_mix(sesa_mix(sesa_mix(value_seed ^ block) ^ t) ^ k)
 *                with sesa_mix(x) = splitmix64 finaliser of (x + 0x9E3779B97F4A7C15).
 * Output order is the paper's canonical sequential schedule: ascending block, then ascending
 * interval, then ascending thread t, then descriptor index (program order), then k. */
typedef struct {
  uint64_t base;
  int64_t bstride, tstride, istride;
  uint64_t value_seed;
  uint32_t block_lo, block_hi; /* blocks [block_lo, block_hi)                        */
  uint32_t nthreads;           /* threads per block of the flow: t in [0, nthreads)  */
  uint32_t interval;
  uint32_t pmask, pval;
  uint32_t pmod, prem;
  uint32_t plo, phi;
  uint32_t fkind, fc, fm;
  uint32_t count;
  uint16_t size;
  uint8_t space, rw;
  uint32_t flags;
} sesa_flow; /* 104 bytes */

enum { SESA_F_ID = 0, SESA_F_MODADD = 1, SESA_F_XOR = 2, SESA_F_SHR = 3, SESA_F_ROW2D = 4 };
enum { SESA_FLOW_CONST_VALUE = 1 };

typedef struct sesa_trace sesa_trace; /* opaque; owns device scratch and the last race list */

/* Per-kernel timing of the last sesa_race_check (only when profiling is enabled). */
typedef struct {
  char name[32];        /* kernel family, e.g. "onesweep_pass"                                            */
  uint32_t launches;    /* launches in the last check                                                      */
  float ms;             /* summed CUDA-event time of those launches on the check's stream                  */
  double bytes;         /* algorithmic bytes those launches must move (DESIGN.md §6 per-unit figures)       */
} sesa_kernel_stat;

typedef struct {
  uint64_t n_records, n_entries, n_races;
  uint64_t n_multi;         /* entries at locations touched >= 2 times (the only ones that can race) — with
                               wbit_filter, minus (most) entries of locations that no entry writes   */
  uint32_t sort_bits, pos_bits, digit_bits, sort_passes; /* key layout chosen by the extents pass   */
  uint32_t sorted_input;    /* records were (block, interval)-ordered                               */
  uint32_t launches;        /* kernels launched by the last check (all families)                    */
  uint32_t crossing_tiles;  /* conflict tiles with a location run crossing a tile boundary          */
  uint32_t n_stats;         /* valid entries of sesa_trace_kernel_stats                             */
  uint32_t fused_first_pass;/* key extract and the first sort pass ran as one kernel   */
  uint32_t bucket_path;     /* the sort ran only over the two high digits and each chunk of 2^15 granules was
                               resolved by a shared-memory bitmap ("bucket path")             */
  uint32_t wbit_filter;     /* the compaction also dropped read-only locations (a write bit in the sort key,
                               DESIGN.md §5.6; chosen by a sample of the sorted keys)                        */
} sesa_check_info;

/* Create a single-GPU handle on the current CUDA device.  cfg is validated (EINVAL on warp_size 0,
 * lockstep > 1, granularity not a power of 2 or > 4096, unknown flags bits).  *out = NULL on error. */
sesa_status sesa_trace_create(const sesa_config *cfg, sesa_trace **out);

/* Collective: create a handle that is rank `rank` of `world` (one process per GPU).  nccl_unique_id is the
 * 128-byte ncclUniqueId produced by rank 0 (sesa_nccl_unique_id) and broadcast by the caller (e.g. with
 * torch.distributed).  Records are then exchanged by location hash. */
sesa_status sesa_trace_create_dist(const sesa_config *cfg, int rank, int world, const uint8_t nccl_unique_id[128],
                                   sesa_trace **out);
/* Fill a fresh ncclUniqueId (rank 0 only). */
sesa_status sesa_nccl_unique_id(uint8_t out_id[128]);

/* Race-check n records in DEVICE memory (borrowed; must stay valid until return).  Record i has global index
 * index_base + i.  Enqueues on cuda_stream and returns when the race list is complete (it synchronises the
 * stream).  A host pointer is EINVAL.  n == 0 is valid (no races).  Distributed handles: collective; every
 * rank passes its shard and the exclusive prefix of shard sizes as index_base; rank 0 receives the merged
 * list, identical to a 1-GPU check of the concatenated trace; other ranks receive 0 races. */
sesa_status sesa_race_check(sesa_trace *t, const sesa_access *d_records, uint64_t n, uint64_t index_base,
                            void *cuda_stream);

/* Test/diagnostic entry: the distributed check of sesa_race_check with `world` (<= 8) VIRTUAL ranks on the
 * current GPU — the same kernels and data flow as the NCCL path (partition by location owner, key exchange,
 * record fetch, race gather), with the exchanges done by device copies.  Rank r owns records
 * [offs[r], offs[r+1]) of d_records (offs has world+1 entries, offs[0] = 0).  On return *out is a handle holding
 * the merged race list (read it with sesa_races_get; destroy it with sesa_trace_destroy).  The result must equal
 * a single-GPU check of the same records (tests/test_gpu_dist.py). */
sesa_status sesa_race_check_loopback(const sesa_config *cfg, const sesa_access *d_records, const uint64_t *offs,
                                     int world, uint64_t index_base, void *cuda_stream, sesa_trace **out);

/* Same, for records in HOST memory: the library copies them to the device inside the call — one DMA when
 * h_records is page-locked (cudaHostAlloc / registered), else in 64 MiB chunks through two page-locked staging
 * buffers (the host copy of a chunk overlaps the DMA of the previous one).  The device copy is owned by the
 * handle (grow-only).  This is the end-to-end entry point. */
sesa_status sesa_race_check_host(sesa_trace *t, const sesa_access *h_records, uint64_t n, uint64_t index_base,
                                 void *cuda_stream);

/* Multi-launch trace (Table IV's per-kernel verdicts P:467 come from programs that launch
 * several kernels): records [launch_offsets[e], launch_offsets[e+1]) were made by kernel launch e, e < n_launches
 * (launch_offsets: HOST array of n_launches + 1 entries, launch_offsets[0] = 0, non-decreasing,
 * launch_offsets[n_launches] = n; else EINVAL).  The launches of one trace run one after another on the stream,
 * so accesses of different launches are ordered — like accesses separated by a barrier — and never race
 * (reading R23): the launch is part of the location, and each race record names it in `epoch`.
 * Record i keeps its global index index_base + i.  The OOB report covers every launch.  Single-GPU handles only
 * (EINVAL on distributed handles). */
sesa_status sesa_race_check_launches(sesa_trace *t, const sesa_access *d_records, uint64_t n,
                                     const uint64_t *launch_offsets, uint32_t n_launches, uint64_t index_base,
                                     void *cuda_stream);

/* Precise warp model.  P:281 (§IV-B): "two intra-warp threads can race only if they
 * simultaneously write to the same shared variable at the same instruction.  In case of divergence, we execute
 * the two sides sequentially ... [and] enumerate both orders"; P:87 (§II): a divergent read/write races "no matter
 * whether t1 and t2 are within a warp".  Every record gets an extension: pc = the static instruction of the
 * access; div = 0 if its warp was convergent there, else (branch instance << 1 | side) of the innermost divergent
 * branch region containing it (instances numbered by the producer, unique per warp execution of a branch).
 * With cfg.lockstep = 1, two records of different threads in one block, interval and warp race only if
 *   (a) they lie on the two sides of one branch instance (same div >> 1, different div & 1, both != 0) — then by
 *       rules (1)-(4) and (6) as without lockstep — or
 *   (b) both write (plain or atomic, not both atomic) at the same pc — a W/W race, benign filter (6) applies;
 * this replaces rule (5) (reading R24).  Pairs of different warps or blocks follow the ordinary rules.
 * With every pc equal and every div 0 the model is rule (5).  lockstep = 0: d_ext is ignored.
 * d_ext: DEVICE array of n sesa_access_ext (8 bytes each), borrowed like d_records.  Single-GPU handles, no
 * SESA_FLAG_REPORT_BENIGN (EINVAL). */
typedef struct {
  uint32_t pc;   /* static instruction id                                                                     */
  uint32_t div;  /* 0 = convergent; else (branch instance << 1) | side                                        */
} sesa_access_ext;

sesa_status sesa_race_check_warp(sesa_trace *t, const sesa_access *d_records, const sesa_access_ext *d_ext,
                                 uint64_t n, uint64_t index_base, void *cuda_stream);

/* Copy the last race list to host memory (caller-owned).  cap == 0: only *n_races is set.  cap < count:
 * copies cap races, sets *n_races = count, returns SESA_ETRUNC.  ESTATE when no successful check. */
sesa_status sesa_races_get(sesa_trace *t, sesa_race *host_out, uint64_t cap, uint64_t *n_races);

/* Device pointer to the last race list (owned by the handle, valid until the next check or destroy). */
sesa_status sesa_races_device(sesa_trace *t, const sesa_race **d_races, uint64_t *n_races);

/* Expand n_flows descriptors (device memory) into records at d_out (device, capacity cap records).
 * *n_out = number of records the descriptors produce; if it exceeds cap nothing is written and SESA_ETRUNC
 * is returned (call with cap = 0 to size the output).  Synchronises cuda_stream. */
sesa_status sesa_expand(sesa_trace *t, const sesa_flow *d_flows, uint64_t n_flows, sesa_access *d_out, uint64_t cap,
                        uint64_t *n_out, void *cuda_stream);

/* Descriptor-level check: the race list of the trace that sesa_expand(d_flows) describes —
 * identical, witnesses included (indices in the canonical expansion order), to expanding and checking it — decided
 * per pair of descriptors first.  The paper instantiates two flows' accesses at two symbolic threads t1 != t2 and
 * asks a solver whether an address can coincide (§IV-A, §IV-B); here interval arithmetic on
 * the address functions (base + bstride*block + tstride*f(t) + istride*k, f in {id, modadd, xor, shr, row2d})
 * proves pairs race-free without instantiating any thread: disjoint granule ranges, read/read, atomic/atomic, no
 * common block or interval where ordering requires one, and plain-write descriptors whose instances never share a
 * granule (injective f, strides beyond size + G - 1).  Only descriptors left in some undecided pair are
 * instantiated and checked.  d_flows: DEVICE array.  Synchronises the stream. */
sesa_status sesa_race_check_flows(sesa_trace *t, const sesa_flow *d_flows, uint64_t n_flows, void *cuda_stream);

typedef struct {
  uint64_t n_flows;           /* descriptors given                                                         */
  uint64_t n_flows_checked;   /* descriptors left in an undecided pair (instantiated)                      */
  uint64_t n_records;         /* records the descriptors describe (the full expansion)                     */
  uint64_t n_records_checked; /* records instantiated and checked                                          */
} sesa_flow_check_info;
sesa_status sesa_flow_check_get(const sesa_trace *t, sesa_flow_check_info *out);

/* Profiling: when enabled, every kernel of a check is bracketed by CUDA events on the check's stream. */
sesa_status sesa_trace_set_profiling(sesa_trace *t, int enable);
sesa_status sesa_trace_info(const sesa_trace *t, sesa_check_info *out);
sesa_status sesa_trace_kernel_stats(const sesa_trace *t, sesa_kernel_stat *out, uint32_t cap, uint32_t *n_out);

/* ---- Out-of-bound check (Table IV "OOB" P:467, the histo_final OOB of Fig. 9).
 * A memory region is an allocation {base, size} of one space (the paper's "size of the memory region the
 * pointer ... refers to").  With regions registered for a space, a valid record of that space is OUT OF
 * BOUND iff no registered region R of its space contains all its bytes: R.base <= addr and
 * addr + size <= R.base + R.size.  Spaces without registered regions are not checked.  The check runs inside
 * the validation pass of every sesa_race_check (no extra pass over the records); it does not change the race
 * list.  The witness is canonical: the lowest (index_base-adjusted) record index among the OOB records. */
typedef struct {
  uint64_t base;  /* first byte (SHARED: offset in the block's window; GLOBAL: device byte address)          */
  uint64_t size;  /* bytes, >= 1; base + size must not wrap                                                 */
  uint32_t space; /* SESA_SPACE_*                                                                          */
  uint32_t reserved; /* zero                                                                               */
} sesa_region;

/* Register n (<= 1024) regions (host array, copied); n == 0 clears them.  EINVAL on space > 1, size 0,
 * wrap-around, reserved != 0, or two regions of one space that overlap. */
sesa_status sesa_trace_set_regions(sesa_trace *t, const sesa_region *regions, uint32_t n);

typedef struct {
  uint64_t n_oob;       /* OOB records in the last check                                                   */
  uint64_t first_index; /* lowest OOB record index (index_base-adjusted); UINT64_MAX if none                */
  sesa_access first;    /* that record (zero if none)                                                       */
} sesa_oob_report;

/* The OOB report of the last successful check (ESTATE before one).  Distributed handles: every rank holds the
 * report merged over all ranks (each rank checks its own shard against its own registered regions). */
sesa_status sesa_oob_get(const sesa_trace *t, sesa_oob_report *out);

void sesa_trace_destroy(sesa_trace *t); /* NULL-safe; frees all device scratch */
const char *sesa_status_str(sesa_status s);
const char *sesa_last_error(const sesa_trace *t); /* "" if none; valid until the next call on t */
int sesa_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SESA_H */
