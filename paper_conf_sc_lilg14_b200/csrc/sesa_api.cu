// sesa_api.cu — the C ABI of include/sesa.h: handle, validation, buffer management and the orchestration of
// the sm_100a pipeline.  Host code only; every step of the race check runs in the kernels of
// k_*.cu.  There is no CPU fallback: without a CUDA device every call fails with SESA_ECUDA.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/sesa.h"
#include "kernels.cuh"
#include "sesa_internal.h"

using namespace sesa;

static_assert(sizeof(sesa_access) == 32, "sesa_access");
static_assert(sizeof(sesa_race) == 40, "sesa_race");
static_assert(sizeof(sesa_flow) == 104, "sesa_flow");

// ------------------------------------------------------------------------------------------------ helpers
static u32 bits_of(u64 x) { return x == 0 ? 0u : 64u - (u32)__builtin_clzll(x); }

void sesa_trace::fail(sesa_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  err = buf;
  status = s;
}

bool sesa_trace::cuda_ok(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return true;
  fail(e == cudaErrorMemoryAllocation ? SESA_ENOMEM : SESA_ECUDA, "%s: %s", what, cudaGetErrorString(e));
  cudaGetLastError();
  return false;
}

bool sesa_trace::grow(DevBuf& b, size_t bytes, const char* what) {
  if (b.cap >= bytes) return true;
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.cap = 0;
  size_t want = std::max<size_t>(bytes, 256);
  if (!cuda_ok(cudaMalloc(&b.p, want), what)) return false;
  b.cap = want;
  return true;
}

bool sesa_trace::grow_keep(DevBuf& b, size_t bytes, size_t used, const char* what) {
  if (b.cap >= bytes) return true;
  void* p = nullptr;
  const size_t want = std::max<size_t>(bytes, 256);
  if (!cuda_ok(cudaMalloc(&p, want), what)) return false;
  if (used && b.p && !cuda_ok(cudaMemcpyAsync(p, b.p, std::min(used, b.cap), cudaMemcpyDeviceToDevice, stream), what))
    return false;
  if (b.p) cudaFree(b.p);  // (synchronises: the copy has completed)
  b.p = p;
  b.cap = want;
  return true;
}

void sesa_trace::free_all() {
  for (DevBuf* b : all_bufs())
    if (b->p) cudaFree(b->p), b->p = nullptr, b->cap = 0;
  for (auto& e : ev_pool) cudaEventDestroy(e);
  ev_pool.clear();
  if (h_pinned) cudaFreeHost(h_pinned), h_pinned = nullptr;
}

// ------------------------------------------------------------------------------------------------ profiling
// kernels one LAUNCH family issues (memsets excluded): info.launches counts kernels, not families
static unsigned kernels_of(const char* name) {
  static const struct {
    const char* n;
    unsigned k;
  } tab[] = {{"tile_offsets", 3}, {"compact", 4}, {"carry", 3}, {"alltoall", 0}, {"flow_pairs", 2},
                 {"owner_partition", 4}, {"conflict_cross", 2}, {"conflict_y", 2}};  // alltoall: NCCL's kernels
  for (const auto& e : tab)
    if (!strcmp(e.n, name)) return e.k;
  return 1;
}

void sesa_trace::launch_begin(const char* name) {
  launches += kernels_of(name);
  prof_last = name;
  if (!profiling) return;
  ProfRec r;
  r.name = name;
  r.ev0 = next_event();
  cudaEventRecord(r.ev0, stream);
  prof.push_back(r);
}
void sesa_trace::launch_end(double bytes) {
  static const bool dbg = getenv("SESA_SYNC_DEBUG") != nullptr;
  if (dbg) {  // pinpoint the failing launch
    cudaError_t e = cudaStreamSynchronize(stream);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) fprintf(stderr, "[sesa debug] after %s: %s\n", prof_last.c_str(), cudaGetErrorString(e));
  }
  if (!profiling) return;
  ProfRec& r = prof.back();
  r.ev1 = next_event();
  r.bytes = bytes;
  cudaEventRecord(r.ev1, stream);
}
cudaEvent_t sesa_trace::next_event() {
  if (ev_used == ev_pool.size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    ev_pool.push_back(e);
  }
  return ev_pool[ev_used++];
}
void sesa_trace::collect_prof() {
  stats.clear();
  if (!profiling) return;
  for (auto& r : prof) {
    float ms = 0;
    cudaEventElapsedTime(&ms, r.ev0, r.ev1);
    auto it = std::find_if(stats.begin(), stats.end(), [&](const sesa_kernel_stat& s) { return r.name == s.name; });
    if (it == stats.end()) {
      sesa_kernel_stat s;
      memset(&s, 0, sizeof s);
      snprintf(s.name, sizeof s.name, "%s", r.name.c_str());
      stats.push_back(s);
      it = stats.end() - 1;
    }
    it->launches++;
    it->ms += ms;
    it->bytes += r.bytes;
  }
}

#define LAUNCH(name, bytes, call) \
  do {                            \
    launch_begin(name);           \
    call;                         \
    launch_end(bytes);            \
  } while (0)

// ------------------------------------------------------------------------------------------------ check
bool sesa_trace::sync_check(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_ok(e, what);
  return cuda_ok(cudaStreamSynchronize(stream), what);
}

// Computes the key layout (common.cuh) from the extents summary.  Returns false (ERANGE) if it does not fit.
bool sesa_trace::make_layout(const Summary& S, u64 n) {
  KeyLayout& L = layout;
  memset(&L, 0, sizeof L);
  L.log2G = (u32)__builtin_ctz(cfg.granularity);
  const bool hasS = S.count[0] > 0, hasG = S.count[1] > 0;
  L.both = hasS && hasG;
  L.single_space = hasS ? SP_SHARED : SP_GLOBAL;
  u32 shared_bits = 0, global_bits = 0;
  if (hasS) {
    L.gminS = S.gmin[0];
    L.bminS = S.bmin[0];
    L.iminS = S.imin[0];
    L.gbS = bits_of(S.gmax[0] - S.gmin[0]);
    L.ibS = bits_of((u64)(S.imax[0] - S.imin[0]));
    L.bbS = bits_of((u64)(S.bmax[0] - S.bmin[0]));
    shared_bits = L.gbS + L.ibS + L.bbS;
  }
  if (hasG) {
    L.gminG = S.gmin[1];
    L.bminG = S.bmin[1];
    L.iminG = S.imin[1];
    L.gbG = bits_of(S.gmax[1] - S.gmin[1]);
    if (S.unsorted) {
      L.ibG = bits_of((u64)(S.imax[1] - S.imin[1]));
      L.bbG = bits_of((u64)(S.bmax[1] - S.bmin[1]));
      L.lowG = L.ibG + L.bbG;
    }
    global_bits = L.gbG + L.lowG;
  }
  // shared runs need (block, interval) order too: in the unsorted case they are part of the shared key anyway
  L.sort_bits = std::max(shared_bits, global_bits) + (L.both ? 1u : 0u);
  L.space_shift = L.both ? L.sort_bits - 1 : 0;
  L.pos_bits = std::max(1u, bits_of(n - 1));
  if (L.sort_bits + L.pos_bits > 64) {
    fail(SESA_ERANGE, "key layout needs %u sort bits + %u position bits > 64 (granule span %u bits)", L.sort_bits,
         L.pos_bits, std::max(L.gbS, L.gbG));
    return false;
  }
  return true;
}

void sesa_trace::begin_check(u64 n) {
  status = SESA_OK;
  have_oob = false;
  err.clear();
  have_result = false;
  n_races = 0;
  launches = 0;
  prof.clear();
  ev_used = 0;
  memset(&info, 0, sizeof info);
  info.n_records = n;
}

bool sesa_trace::check_records_ptr(const sesa_access* d_rec, u64 n) {
  if (!d_rec) return fail(SESA_EINVAL, "d_records is NULL"), false;
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, d_rec) != cudaSuccess ||
      (pa.type != cudaMemoryTypeDevice && pa.type != cudaMemoryTypeManaged)) {
    cudaGetLastError();
    return fail(SESA_EINVAL, "d_records is not device memory (use sesa_race_check_host for host buffers)"), false;
  }
  if (n >= (1ull << 31)) return fail(SESA_ERANGE, "n = %llu >= 2^31 records (ABI v1 limit)", (unsigned long long)n), false;
  return true;
}

// step 1: validation + extents of the local records -> h_summary (synchronises)
bool sesa_trace::step_extents(const Rec* rec, u64 n, bool tile_hist, u32* gran_out) {
  const u32 log2G = (u32)__builtin_ctz(cfg.granularity);
  if (!grow(b_summary, sizeof(Summary), "summary")) return false;
  // per-tile raw digit histograms for the fused first pass (worth it only for traces of many tiles)
  have_thist = tile_hist && n >= 32768;
  if (have_thist && !grow(b_thist, ((n + FUSED_TILE - 1) / FUSED_TILE) * RADIX * 4, "tile histograms")) return false;
  // large traces: also the tile histograms of the bucket path's first digit (k_bucket.cu)
  have_thist2 = have_thist && n >= BUCKET_MIN_N;
  if (have_thist2 && !grow(b_thist2, ((n + FUSED_TILE - 1) / FUSED_TILE) * RADIX * 4, "tile histograms")) return false;
  // granule indices for the fused pass go to the key buffer the first sort pass after it writes (b_keys[0])
  if (have_thist && !grow(b_keys[0], n * 8 + 64, "keys")) return false;
  // and the per-record write bits the fused pass puts into the keys (KeyLayout::wbit)
  if (have_thist && !grow(b_wbits, (n + 31) / 32 * 4, "write bits")) return false;
  Summary init;
  memset(&init, 0, sizeof init);
  init.bad_index = ~0ull;
  init.oob_first = ~0ull;
  init.gmin[0] = init.gmin[1] = ~0ull;
  init.bmin[0] = init.bmin[1] = init.imin[0] = init.imin[1] = ~0u;
  h_summary = init;
  if (n == 0) return true;
  if (!cuda_ok(cudaMemcpyAsync(b_summary.p, &h_summary, sizeof(Summary), cudaMemcpyHostToDevice, stream), "summary init"))
    return false;
  const int grid_stream = (int)std::min<u64>((n + 255) / 256, (u64)num_sms * 8);
  // the 32-bit granule array: for the fused first pass (b_keys[0]) or the caller's (distributed owner partition)
  u32* gout = have_thist ? (u32*)b_keys[0].p : gran_out;
  LAUNCH("extents", (gout ? 36.0 : 32.0) * n, launch_extents(rec, n, log2G, (Summary*)b_summary.p,
                                             have_thist ? (u32*)b_thist.p : nullptr, (const Region*)b_regions.p,
                                             n_regions, n_regions_shared, grid_stream, stream, gout,
                                             have_thist2 ? (u32*)b_thist2.p : nullptr,
                                             have_thist ? (u32*)b_wbits.p : nullptr));
  if (!cuda_ok(cudaMemcpyAsync(&h_summary, b_summary.p, sizeof(Summary), cudaMemcpyDeviceToHost, stream), "summary"))
    return false;
  return sync_check("extents");
}

void sesa_trace::set_oob(const sesa_access* d_rec, u64 count, u64 local_first, u64 index_base) {
  memset(&oob, 0, sizeof oob);
  oob.n_oob = count;
  oob.first_index = count ? index_base + local_first : ~0ull;
  if (count) cudaMemcpy(&oob.first, d_rec + local_first, sizeof(sesa_access), cudaMemcpyDeviceToHost);
  have_oob = true;
}

bool sesa_trace::report_bad(const sesa_access* d_rec, u64 local_bad, u64 global_bad) {
  sesa_access r;
  cudaMemcpy(&r, d_rec + local_bad, sizeof r, cudaMemcpyDeviceToHost);
  fail(SESA_EINVAL, "record %llu invalid (space=%u rw=%u size=%u addr=0x%llx)", (unsigned long long)global_bad, r.space,
       r.rw, r.size, (unsigned long long)r.addr);
  return false;
}

// step 2: keys (+ the histograms of every sort digit) of the local records at positions pos_base + i -> b_keys[0]
bool sesa_trace::step_extract(const Rec* rec, u64 n, u64 m, u64 pos_base, bool multi) {
  const KeyLayout& L = layout;
  const u32 npass = (L.sort_bits + RADIX_BITS - 1) / RADIX_BITS;
  const u32 log2G = L.log2G;
  if (!grow(b_keys[0], m * 8 + 64, "keys") || !grow(b_keys[1], m * 8 + 64, "keys") ||
      !grow(b_hist, (size_t)std::max(npass, 1u) * RADIX * 4, "hist") ||
      !grow(b_binbase, (size_t)std::max(npass, 1u) * RADIX * 8, "binbase"))
    return false;
  cudaMemsetAsync(b_hist.p, 0, (size_t)std::max(npass, 1u) * RADIX * 4, stream);
  if (n == 0) return true;
  u64* keys = (u64*)b_keys[0].p;
  const int grid_stream = (int)std::min<u64>((n + 255) / 256, (u64)num_sms * 8);
  if (!multi) {
    LAUNCH("extract", 40.0 * n, launch_extract_1to1(rec, n, L, npass, keys, (u32*)b_hist.p, pos_base, grid_stream, stream));
  } else {
    if (!grow(b_cnt, n * 4, "counts") || !grow(b_off, n * 4, "offsets") || !grow(b_temp, scan_u32_temp_bytes(n), "scan"))
      return false;
    LAUNCH("entry_count", 36.0 * n, launch_entry_count(rec, n, log2G, (u32*)b_cnt.p, stream));
    LAUNCH("scan", 8.0 * n, launch_scan_exclusive_u32((u32*)b_cnt.p, (u32*)b_off.p, n, b_temp.p, stream));
    LAUNCH("extract_multi", 36.0 * n + 8.0 * m,
           launch_extract_multi(rec, n, L, npass, (u32*)b_off.p, keys, (u32*)b_hist.p, pos_base, grid_stream, stream));
  }
  return true;
}

// step 2+3a (fused): keys of the records sorted by the first digit -> b_keys[1], histograms of the other digits
bool sesa_trace::step_extract_fused(const Rec* rec, u64 n) {
  const KeyLayout& L = layout;
  const u32 npass = (L.sort_bits + RADIX_BITS - 1) / RADIX_BITS;
  if (!grow(b_keys[0], n * 8 + 64, "keys") || !grow(b_keys[1], n * 8 + 64, "keys") ||
      !grow(b_hist, (size_t)npass * RADIX * 4, "hist") || !grow(b_binbase, (size_t)npass * RADIX * 8, "binbase") ||
      !grow(b_ftmp, fused_temp_bytes(n), "fused temp"))
    return false;
  cudaMemsetAsync(b_hist.p, 0, (size_t)npass * RADIX * 4, stream);
  if (hist_from_extents) {  // digit p >= 1 = raw granule byte p; the top digit rotated by byte p of gmin
    std::vector<u32> rows((size_t)(npass - 1) * RADIX);
    for (u32 p = 1; p < npass; p++) {
      const u32 r = p == npass - 1 ? (u32)(L.gminG >> (RADIX_BITS * p)) & (RADIX - 1) : 0u;
      for (u32 d = 0; d < (u32)RADIX; d++) rows[(size_t)(p - 1) * RADIX + d] = h_summary.bhist[p - 1][(d + r) & (RADIX - 1)];
    }
    if (!cuda_ok(cudaMemcpyAsync((u32*)b_hist.p + RADIX, rows.data(), rows.size() * 4, cudaMemcpyHostToDevice, stream),
                 "hist rows"))
      return false;
  }
  LAUNCH("tile_offsets", 2.0 * RADIX * 4 * ((n + FUSED_TILE - 1) / FUSED_TILE),
         launch_tile_offsets(n, L, (const u32*)b_thist.p, b_ftmp.p, stream));
  LAUNCH("extract_pass0", 12.0 * n,
         launch_fused_extract_pass0((const u32*)b_keys[0].p, n, L, hist_from_extents ? 1u : npass, b_ftmp.p,
                                    (u64*)b_keys[1].p, (u32*)b_hist.p, stream, 0, false, (const u32*)b_wbits.p));
  return true;
}

// ---- bucket path (k_bucket.cu): decide, then fused pass on key_hi bits [14, 22), one onesweep pass on [22, 30),
// per-chunk bitmap filter + sort of the survivors.  Chosen when the granules spread evenly: a sample of the
// granule array must show no chunk of 2^HYB_CHUNK granules much above the mean (C5); hot regions (C3's bins,
// C4's dist[]) keep the full sort, where almost every entry survives anyway.
bool sesa_trace::bucket_choose(u64 n, u64* gmin_aligned, u32* nbits, u32* nchunks) {
  const Summary& S = h_summary;
  const u32 D = HYB_LO + RADIX_BITS;  // gmin aligned to 2^22: both global digits are raw granule bytes, rotated
  const u64 G0 = S.gmin[1] & ~((1ull << D) - 1ull);
  const u32 nb = bits_of(S.gmax[1] - G0);
  if (nb <= D || nb > HYB_LO + 2 * RADIX_BITS || nb + layout.pos_bits > 64) return false;
  const u32 nc = (u32)(((S.gmax[1] - G0) >> HYB_CHUNK) + 1);
  if (!grow(b_btmp2, bucket_temp_bytes(nc), "bucket temp")) return false;
  // a 64 K sample first: a hot region (C3's bins, C4's `changed`) shows at once; then 4 M samples for the bound
  const double mean = (double)n / nc;
  for (u32 want : {1u << 16, 1u << 22}) {
    u32 hmax = 0, samples = 0;
    LAUNCH("bucket_sample", 4.0 * (double)want, launches += bucket_sample_max((const u32*)b_keys[0].p, (u32)n, (u32)G0, nc,
                                                                             b_btmp2.p, stream, &hmax, &samples, want) - 1);
    if (!sync_check("bucket sample")) return false;
    const double est_max = (double)hmax * (double)n / (double)std::max(1u, samples);
    if (want < (1u << 22) ? est_max > 32.0 * mean + 65536.0 : (est_max > 4.0 * mean + 2048.0 || est_max > (double)(1u << 20)))
      return false;
  }
  *gmin_aligned = G0;
  *nbits = nb;
  *nchunks = nc;
  return true;
}

bool sesa_trace::step_bucket(u64 n, u32 nchunks, u64** comp, u32* m2) {
  const KeyLayout& L = layout;
  // the fused pass's output carries up to 31 sentinels per digit run (32-aligned runs, below)
  if (!grow(b_keys[1], (n + 32 * RADIX) * 8 + 64, "keys") || !grow(b_hist, 2 * RADIX * 4, "hist") ||
      !grow(b_binbase, 2 * RADIX * 8, "binbase") || !grow(b_ftmp, fused_temp_bytes(n), "fused temp") ||
      !grow(b_ctotal, 16, "compact count"))
    return false;
  // digit B (key_hi bits [22, 30)) = raw granule bits [22, 30) rotated by those of gmin: its histogram is the
  // extents' row 3
  std::vector<u32> row(RADIX);
  const u32 r = (u32)(L.gminG >> (HYB_LO + RADIX_BITS)) & (RADIX - 1);
  for (u32 d = 0; d < (u32)RADIX; d++) row[d] = h_summary.bhist[3][(d + r) & (RADIX - 1)];
  if (!cuda_ok(cudaMemcpyAsync((u32*)b_hist.p + RADIX, row.data(), RADIX * 4, cudaMemcpyHostToDevice, stream), "hist"))
    return false;
  cudaMemsetAsync(b_hist.p, 0, RADIX * 4, stream);
  // Both partition passes are unstable (k_bucket.cu).  The second keeps the first one's digit order only if no
  // 32-key row of its input holds two first-digit values: the first pass pads every digit run to a multiple of
  // 32 with ~0 sentinels, which the second pass skips.
  const bool pass2 = *std::max_element(row.begin(), row.end()) != n;  // digit B not trivial
  LAUNCH("tile_offsets", 2.0 * RADIX * 4 * ((n + FUSED_TILE - 1) / FUSED_TILE),
         launch_tile_offsets(n, L, (const u32*)b_thist2.p, b_ftmp.p, stream, HYB_LO,
                             pass2 ? (u64*)b_keys[1].p : nullptr, (u32*)b_ctotal.p + 2));
  u32 mpad = (u32)n;
  if (pass2 && (!cuda_ok(cudaMemcpyAsync(&mpad, (u32*)b_ctotal.p + 2, 4, cudaMemcpyDeviceToHost, stream), "padded") ||
                !sync_check("tile offsets")))
    return false;
  LAUNCH("extract_pass0", 12.0 * n,
         launch_fused_extract_pass0((const u32*)b_keys[0].p, n, L, 1, b_ftmp.p, (u64*)b_keys[1].p, (u32*)b_hist.p,
                                    stream, HYB_LO, true));
  int cur = 1;
  u32 passes = 1;
  if (pass2) {
    LAUNCH("bin_base", 0.0, launch_bin_base((u32*)b_hist.p, (u64*)b_binbase.p, 2, stream));
    const u32 stiles = sort_tiles(mpad);
    if (!grow(b_lookback, (size_t)stiles * RADIX * 8, "lookback") || !grow(b_ctr, 64 * 4, "counters")) return false;
    if (b_lookback.cap != lookback_cleared) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      lookback_cleared = b_lookback.cap;
      epoch = 0;
    }
    cudaMemsetAsync(b_ctr.p, 0, 64 * 4, stream);
    if (++epoch >= 256) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      epoch = 1;
    }
    LAUNCH("partition_pass", 16.0 * n,
           launch_partition_pass((u64*)b_keys[1].p, (u64*)b_keys[0].p, mpad, L.pos_bits + HYB_LO + RADIX_BITS,
                                 (u64*)b_binbase.p + RADIX, (u64*)b_lookback.p, (u32*)b_ctr.p, epoch, stream));
    cur = 0;
    passes++;
  }
  info.sort_passes = passes;
  // per-chunk bitmap filter + sort of the survivors; result (sorted, compacted) back in b_keys[cur]
  LAUNCH("bucket", 8.0 * n,
         launches += launch_bucket_compact((u64*)b_keys[cur].p, (u64*)b_keys[cur ^ 1].p, (u32)n, L.pos_bits, nchunks,
                                           b_btmp2.p, (u32*)b_ctotal.p, stream) - 1);
  *comp = (u64*)b_keys[cur].p;
  if (!cuda_ok(cudaMemcpyAsync(m2, b_ctotal.p, 4, cudaMemcpyDeviceToHost, stream), "bucket count")) return false;
  if (!sync_check("bucket")) return false;
  info.n_multi = *m2;
  return true;
}

// Bucket path on a key array (b_keys[0], m keys of the current layout) — the distributed check's received keys,
// or a single-GPU trace the fused first pass does not cover: an unstable pass on key_hi bits [14, 22) into
// 32-aligned runs (padded bin bases, sentinels), one on [22, 30), the chunk bitmaps.  *used = false (and true
// returned) when the trace is not eligible: the caller sorts in full.
bool sesa_trace::try_bucket_keys(u64 m, u64** comp, u32* m2, bool* used) {
  *used = false;
  const KeyLayout& L = layout;
  if (m < BUCKET_MIN_N || L.both || (L.single_space == SP_GLOBAL && L.lowG) || L.sort_bits <= HYB_LO + RADIX_BITS ||
      L.sort_bits > HYB_LO + 2 * RADIX_BITS || m >= (1ull << 31))
    return true;
  const u32 nc = (u32)((((1ull << L.sort_bits) - 1) >> HYB_CHUNK) + 1);
  if (!grow(b_btmp2, bucket_temp_bytes(nc), "bucket temp")) return false;
  const double mean = (double)m / nc;
  for (u32 want : {1u << 16, 1u << 22}) {
    u32 hmax = 0, samples = 0;
    LAUNCH("bucket_sample", 8.0 * (double)want,
           launches += bucket_sample_keys_max((const u64*)b_keys[0].p, (u32)m, L.pos_bits + HYB_CHUNK, nc, b_btmp2.p,
                                              stream, &hmax, &samples, want) - 1);
    if (!sync_check("bucket sample")) return false;
    const double est_max = (double)hmax * (double)m / (double)std::max(1u, samples);
    if (want < (1u << 22) ? est_max > 32.0 * mean + 65536.0 : (est_max > 4.0 * mean + 2048.0 || est_max > (double)(1u << 20)))
      return true;
  }
  info.bucket_path = 1;
  if (!grow(b_keys[1], (m + 32 * RADIX) * 8 + 64, "keys") || !grow(b_hist, 2 * RADIX * 4, "hist") ||
      !grow(b_binbase, 2 * RADIX * 8, "binbase") || !grow(b_ctotal, 16, "bucket count"))
    return false;
  cudaMemsetAsync(b_hist.p, 0, 2 * RADIX * 4, stream);
  LAUNCH("hist", 8.0 * m, launch_hist_keys_shift((const u64*)b_keys[0].p, (u32)m, 2, L.pos_bits + HYB_LO,
                                                 (u32*)b_hist.p, stream));
  std::vector<u32> rowB(RADIX);
  if (!cuda_ok(cudaMemcpyAsync(rowB.data(), (u32*)b_hist.p + RADIX, RADIX * 4, cudaMemcpyDeviceToHost, stream), "hist") ||
      !sync_check("bucket hist"))
    return false;
  const bool pass2 = *std::max_element(rowB.begin(), rowB.end()) != m;
  u32 mpad = (u32)m;
  if (pass2) {  // 32-aligned digit runs (sentinels in the pad slots) for the second, unstable pass
    LAUNCH("bin_base", 0.0, launch_padded_bin_base((const u32*)b_hist.p, (u64*)b_binbase.p, (u64*)b_keys[1].p,
                                                   (u32*)b_ctotal.p + 2, stream));
    LAUNCH("bin_base", 0.0, launch_bin_base((const u32*)b_hist.p + RADIX, (u64*)b_binbase.p + RADIX, 1, stream));
    if (!cuda_ok(cudaMemcpyAsync(&mpad, (u32*)b_ctotal.p + 2, 4, cudaMemcpyDeviceToHost, stream), "padded") ||
        !sync_check("padded bins"))
      return false;
  } else {
    LAUNCH("bin_base", 0.0, launch_bin_base((const u32*)b_hist.p, (u64*)b_binbase.p, 1, stream));
  }
  const u32 stiles = sort_tiles(std::max<u64>(mpad, m));
  if (!grow(b_lookback, (size_t)stiles * RADIX * 8, "lookback") || !grow(b_ctr, 64 * 4, "counters")) return false;
  if (b_lookback.cap != lookback_cleared) {
    cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
    lookback_cleared = b_lookback.cap;
    epoch = 0;
  }
  cudaMemsetAsync(b_ctr.p, 0, 64 * 4, stream);
  for (int pass = 0; pass < (pass2 ? 2 : 1); pass++) {
    if (++epoch >= 256) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      epoch = 1;
    }
    LAUNCH("partition_pass", 16.0 * m,
           launch_partition_pass((u64*)b_keys[pass].p, (u64*)b_keys[pass ^ 1].p, pass ? mpad : (u32)m,
                                 L.pos_bits + HYB_LO + pass * RADIX_BITS, (u64*)b_binbase.p + pass * RADIX,
                                 (u64*)b_lookback.p, (u32*)b_ctr.p + pass, epoch, stream, pass == 1));
  }
  info.sort_passes = pass2 ? 2 : 1;
  const int cur = pass2 ? 0 : 1;
  LAUNCH("bucket", 8.0 * m,
         launches += launch_bucket_compact((u64*)b_keys[cur].p, (u64*)b_keys[cur ^ 1].p, (u32)m, L.pos_bits, nc,
                                           b_btmp2.p, (u32*)b_ctotal.p, stream) - 1);
  *comp = (u64*)b_keys[cur].p;
  if (!cuda_ok(cudaMemcpyAsync(m2, b_ctotal.p, 4, cudaMemcpyDeviceToHost, stream), "bucket count") ||
      !sync_check("bucket"))
    return false;
  info.n_multi = *m2;
  *used = true;
  return true;
}

// ---- the bucket path with its first partition fused into the extents pass (k_extract.cu "Extents fused with the
// bucket path's first partition"): predicted by a sample of 2^18 records before any pass (global, one granule,
// (block, interval)-ordered, granule span 2^22 .. 2^30, even chunks); then checked exactly on the pass's summary.
// *used = false (and true returned) when not predicted or not eligible: the caller runs the ordinary path.
bool sesa_trace::try_extents_part(const Rec* rec, u64 n, u64 index_base, u64** comp, u32* m2, bool* used) {
  *used = false;
  presample_hot = false;
  if (n < BUCKET_MIN_N || n >= (1ull << 31) || n_regions) return true;
  const u32 log2G = (u32)__builtin_ctz(cfg.granularity);
  {  // a peek at the first 64 records (one small copy): a shared or two-granule record there rules the path out
     // before any sampling kernel (C2 starts with its shared tiles)
    sesa_access head[64];
    const u64 k = std::min<u64>(64, n);
    if (!cuda_ok(cudaMemcpyAsync(head, rec, k * sizeof(sesa_access), cudaMemcpyDeviceToHost, stream), "peek") ||
        !sync_check("peek"))
      return false;
    for (u64 i = 0; i < k; i++) {
      const u64 g0 = head[i].addr >> log2G, g1 = (head[i].addr + (u64)head[i].size - 1ull) >> log2G;
      if (head[i].space != SP_GLOBAL || head[i].size == 0 || g0 != g1) return true;
    }
  }
  if (!grow(b_xtmp, presample_temp_bytes() + 256, "presample") || !grow(b_xsmall, 4096, "regions")) return false;
  // two stages (bucket_choose's bounds): 2^16 samples reject most other traces at once — a shared or
  // multi-granule record, an inversion, a hot region (C2-C4) — then 2^18 samples for the tight chunk bound
  // (C5: ~8 samples per chunk, the sampled maximum ~2.5x the mean: well inside the 4x bound)
  for (u32 want : {1u << 16, 1u << 18}) {
    unsigned long long ext[4] = {1, 0, 0, 0};
    u32 samples = 0;
    LAUNCH("presample", 64.0 * want, launch_presample(rec, (u32)n, log2G, want, b_xtmp.p, ext, &samples, stream));
    if (!sync_check("presample")) return false;
    if (ext[0] || ext[1] > ext[2]) return true;  // a sampled record is shared, multi-granule, invalid or out of order
    const u64 G0 = ext[1] & ~((1ull << (HYB_LO + RADIX_BITS)) - 1ull);
    const u32 nb = bits_of(ext[2] - G0);
    if (nb <= HYB_LO + RADIX_BITS || nb > HYB_LO + 2 * RADIX_BITS) return true;
    const double mean = (double)n / (double)(((ext[2] - G0) >> HYB_CHUNK) + 1);
    const double est_max = (double)ext[3] * (double)n / (double)std::max(1u, samples);
    if (want < (1u << 18) ? est_max > 32.0 * mean + 65536.0
                          : (est_max > 4.0 * mean + 2048.0 || est_max > (double)(1u << 20))) {
      presample_hot = true;  // (bucket_choose's bounds on the same records: it need not sample again)
      return true;
    }
  }
  // the pass
  const u32 pos_bits = std::max(1u, bits_of(n - 1));
  const u64 cap = extents_part_cap(n);
  if (!grow(b_summary, sizeof(Summary), "summary") || !grow(b_keys[1], (size_t)RADIX * cap * 8 + 64, "keys") ||
      !grow(b_keys[0], n * 8 + 64, "keys"))
    return false;
  Summary init;
  memset(&init, 0, sizeof init);
  init.bad_index = ~0ull;
  init.oob_first = ~0ull;
  init.gmin[0] = init.gmin[1] = ~0ull;
  init.bmin[0] = init.bmin[1] = init.imin[0] = init.imin[1] = ~0u;
  u32* gfill = (u32*)b_xsmall.p;
  u32* over = gfill + RADIX;
  if (!cuda_ok(cudaMemcpyAsync(b_summary.p, &init, sizeof(Summary), cudaMemcpyHostToDevice, stream), "summary init"))
    return false;
  cudaMemsetAsync(gfill, 0, (RADIX + 8) * 4, stream);
  XPArgs X{rec, (u32)n, log2G, pos_bits, (Summary*)b_summary.p, (u64*)b_keys[1].p, cap, gfill, over};
  LAUNCH("extents", 40.0 * n, launch_extents_part(X, stream));
  std::vector<u32> fill(RADIX + 1);
  if (!cuda_ok(cudaMemcpyAsync(&h_summary, b_summary.p, sizeof(Summary), cudaMemcpyDeviceToHost, stream), "summary") ||
      !cuda_ok(cudaMemcpyAsync(fill.data(), gfill, (RADIX + 1) * 4, cudaMemcpyDeviceToHost, stream), "fills") ||
      !sync_check("extents"))
    return false;
  const Summary& S = h_summary;
  if (S.bad_index != ~0ull) return report_bad(reinterpret_cast<const sesa_access*>(rec), S.bad_index, S.bad_index);
  const u64 G0 = S.gmin[1] & ~((1ull << (HYB_LO + RADIX_BITS)) - 1ull);
  const u32 nb = S.count[1] == n ? bits_of(S.gmax[1] - G0) : 0u;
  if (fill[RADIX] || S.count[0] || S.multi || S.entries != n || S.unsorted || nb <= HYB_LO + RADIX_BITS ||
      nb > HYB_LO + 2 * RADIX_BITS || nb + pos_bits > 64)
    return true;  // not the bucket path after all (or a region overflowed): the ordinary path from the start
  set_oob(reinterpret_cast<const sesa_access*>(rec), 0, 0, index_base);
  info.n_entries = n;
  info.sorted_input = 1;
  if (!make_layout(S, n)) return false;
  KeyLayout& L = layout;
  L.gminG = G0;
  L.gbG = nb;
  L.sort_bits = nb;
  info.sort_bits = nb;
  info.pos_bits = L.pos_bits;
  info.digit_bits = RADIX_BITS;
  info.fused_first_pass = 1;
  info.bucket_path = 1;
  info.sort_passes = 2;
  // second pass: digit B = key_hi bits [22, 30) (the raw bits rotated by G0's), over the regions in digit-A order
  std::vector<u32> row(RADIX);
  const u32 r = (u32)(G0 >> (HYB_LO + RADIX_BITS)) & (RADIX - 1);
  for (u32 d = 0; d < (u32)RADIX; d++) row[d] = S.bhist[3][(d + r) & (RADIX - 1)];
  // tiles per region from the fullest region (C5: ~1.5% of the tiles are empty or partial)
  const u32 tpr = (*std::max_element(fill.begin(), fill.begin() + RADIX) + PART_TILE_KEYS - 1) / PART_TILE_KEYS;
  const u32 tiles = tpr * RADIX;
  if (!grow(b_hist, 2 * RADIX * 4, "hist") || !grow(b_binbase, 2 * RADIX * 8, "binbase") ||
      !grow(b_ctotal, 16, "bucket count") || !grow(b_lookback, (size_t)tiles * RADIX * 8, "lookback") ||
      !grow(b_ctr, 64 * 4, "counters"))
    return false;
  if (!cuda_ok(cudaMemcpyAsync(b_hist.p, row.data(), RADIX * 4, cudaMemcpyHostToDevice, stream), "hist"))
    return false;
  LAUNCH("bin_base", 0.0, launch_bin_base((const u32*)b_hist.p, (u64*)b_binbase.p, 1, stream));
  if (b_lookback.cap != lookback_cleared) {
    cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
    lookback_cleared = b_lookback.cap;
    epoch = 0;
  }
  cudaMemsetAsync(b_ctr.p, 0, 64 * 4, stream);
  if (++epoch >= 256) {
    cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
    epoch = 1;
  }
  LAUNCH("partition_pass", 16.0 * n,
         launch_partition_regions((const u64*)b_keys[1].p, (u64*)b_keys[0].p, tpr, L.pos_bits + HYB_LO + RADIX_BITS,
                                  (const u64*)b_binbase.p, (u64*)b_lookback.p, (u32*)b_ctr.p, epoch, gfill, cap,
                                  L.pos_bits, (u32)(G0 & ((1ull << 30) - 1ull)), stream));
  // per-chunk bitmap filter + sort of the survivors (k_bucket.cu)
  const u32 nc = (u32)(((S.gmax[1] - G0) >> HYB_CHUNK) + 1);
  if (!grow(b_btmp2, bucket_temp_bytes(nc), "bucket temp")) return false;
  LAUNCH("bucket", 8.0 * n,
         launches += launch_bucket_compact((u64*)b_keys[0].p, (u64*)b_keys[1].p, (u32)n, L.pos_bits, nc, b_btmp2.p,
                                           (u32*)b_ctotal.p, stream) - 1);
  *comp = (u64*)b_keys[0].p;
  if (!cuda_ok(cudaMemcpyAsync(m2, b_ctotal.p, 4, cudaMemcpyDeviceToHost, stream), "bucket count") ||
      !sync_check("bucket"))
    return false;
  info.n_multi = *m2;
  *used = true;
  return true;
}

// step 2' (distributed): histograms of keys that arrived from the exchange (already in b_keys[0])
bool sesa_trace::step_hist(u64 m) {
  const u32 npass = (layout.sort_bits + RADIX_BITS - 1) / RADIX_BITS;
  if (!grow(b_hist, (size_t)std::max(npass, 1u) * RADIX * 4, "hist") ||
      !grow(b_binbase, (size_t)std::max(npass, 1u) * RADIX * 8, "binbase"))
    return false;
  cudaMemsetAsync(b_hist.p, 0, (size_t)std::max(npass, 1u) * RADIX * 4, stream);
  LAUNCH("hist", 8.0 * m, launch_hist_keys_shift((const u64*)b_keys[0].p, (u32)m, npass, layout.pos_bits,
                                                 (u32*)b_hist.p, stream));
  return true;
}

// step 3: LSD onesweep passes over the non-trivial digits of b_keys[0] (m keys); result in b_keys[*cur]
bool sesa_trace::step_sort(u64 m, int* cur_out, u32 first_pass, int cur0) {
  const KeyLayout& L = layout;
  const u32 npass = (L.sort_bits + RADIX_BITS - 1) / RADIX_BITS;
  std::vector<u32> hist((size_t)npass * RADIX);
  if (npass && m) {
    if (!cuda_ok(cudaMemcpyAsync(hist.data(), b_hist.p, hist.size() * 4, cudaMemcpyDeviceToHost, stream), "hist"))
      return false;
    LAUNCH("bin_base", 0.0, launch_bin_base((u32*)b_hist.p, (u64*)b_binbase.p, npass, stream));
  }
  if (!sync_check("extract")) return false;
  const u32 stiles = sort_tiles(m);
  if (npass && m) {
    if (!grow(b_lookback, (size_t)stiles * RADIX * 8, "lookback") || !grow(b_ctr, 64 * 4, "counters")) return false;
    if (b_lookback.cap != lookback_cleared) {  // fresh allocation: clear once, epochs do the rest
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      lookback_cleared = b_lookback.cap;
      epoch = 0;
    }
    cudaMemsetAsync(b_ctr.p, 0, 64 * 4, stream);
  }
  int cur = cur0;
  u32 passes_run = first_pass;
  for (u32 p = first_pass; p < npass && m; p++) {
    const u32* h = hist.data() + (size_t)p * RADIX;
    if (*std::max_element(h, h + RADIX) == m) continue;  // trivial digit: every key has the same value
    if (++epoch >= 256) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      epoch = 1;
    }
    LAUNCH("onesweep_pass", 16.0 * m,
           launch_onesweep((u64*)b_keys[cur].p, (u64*)b_keys[cur ^ 1].p, nullptr, nullptr, (u32)m,
                           L.pos_bits + L.wbit + p * RADIX_BITS, (u64*)b_binbase.p + (size_t)p * RADIX, (u64*)b_lookback.p,
                           (u32*)b_ctr.p + passes_run, epoch, stream));
    cur ^= 1;
    passes_run++;
  }
  info.sort_passes = passes_run;
  *cur_out = cur;
  return true;
}

// step 4: keep entries of locations touched >= 2 times (into the other key buffer) -> (*comp, *m2)
bool sesa_trace::step_compact(int cur, u64 m, u64** comp, u32* m2) {
  // the sorted keys are dead after compaction: the result is concatenated back into their buffer
  *comp = (u64*)b_keys[cur].p;
  *m2 = 0;
  if (m == 0) return true;
  if (!grow(b_ctmp, compact_temp_bytes(m), "compact temp") || !grow(b_ctotal, 16, "compact count")) return false;
  // with the write bit: drop read-only locations too, if a sample of the sorted keys says it pays
  bool filter = false;
  if (layout.wbit) LAUNCH("compact_sample", 8.0 * 32 * 16384,
                          filter = compact_filter_pays((const u64*)b_keys[cur].p, (u32)m, layout, b_ctotal.p, stream));
  info.wbit_filter = filter ? 1 : 0;
  LAUNCH("compact", 8.0 * m, *comp = launch_compact_multi((const u64*)b_keys[cur].p, (u32)m, layout,
                                                          (u64*)b_keys[cur ^ 1].p, (u64*)b_keys[cur].p, b_ctmp.p,
                                                          (u32*)b_ctotal.p, stream, filter));
  if (!cuda_ok(cudaMemcpyAsync(m2, b_ctotal.p, 4, cudaMemcpyDeviceToHost, stream), "compact count")) return false;
  if (!sync_check("compact")) return false;
  info.n_multi = *m2;
  return true;
}

// step 5: conflict tiles (+ crossing carries) over the m2 compacted entries -> unsorted races (b_races, b_rkeys[0],
// b_rvals[0]); n_races set.  Records come by position (rec - rec_pos_base) or entry-aligned (rec_entry).
bool sesa_trace::step_conflict(const u64* comp, u32 m2, const Rec* rec, u32 rec_pos_base, const Rec* rec_entry,
                               u64 index_base) {
  n_races = 0;
  if (m2 == 0) return true;
  const u32 ctiles = conflict_tiles(m2);
  u32 race_cap = (u32)std::min<u64>(std::max<u64>(race_cap_hint, 1u << 16), 2 * (u64)m2 + 16);
  for (int attempt = 0; attempt < 3; attempt++) {
    if (!grow(b_tflags, ctiles, "tile flags") || !grow(b_part, (size_t)ctiles * sizeof(AggQuad), "partials") ||
        !grow(b_carry, (size_t)ctiles * sizeof(AggQuad), "carries") || !grow(b_owner, (size_t)ctiles * 4, "owner") ||
        !grow(b_slots, (size_t)ctiles * sizeof(Slot), "slots") || !grow(b_cross, (size_t)ctiles * 4, "cross") ||
        !grow(b_ccount, 16, "ccount") || !grow(b_races, (size_t)race_cap * sizeof(RaceOut), "races") ||
        !grow(b_rkeys[0], (size_t)race_cap * 8, "race keys") || !grow(b_rkeys[1], (size_t)race_cap * 8, "race keys") ||
        !grow(b_rvals[0], (size_t)race_cap * 4, "race vals") || !grow(b_rvals[1], (size_t)race_cap * 4, "race vals") ||
        !grow(b_carrytmp, carry_temp_bytes(ctiles), "carry temp") ||
        !grow(b_tstart, ((size_t)ctiles + 1) * 4, "tile starts") || !grow(b_work, (size_t)ctiles * 4, "worklist"))
      return false;
    ConflictArgs A;
    memset(&A, 0, sizeof A);
    A.keys = comp;
    A.m = m2;
    A.rec = rec;
    A.rec_entry = rec_entry;
    A.rec_pos_base = rec_pos_base;
    A.L = layout;
    A.ws = conflict_tdiv > 1 ? 1u : cfg.warp_size;
    A.ls = conflict_tdiv > 1 ? 0u : cfg.lockstep;
    A.tdiv = conflict_tdiv;
    A.race_count = (u32*)b_ccount.p;
    A.cross_count = (u32*)b_ccount.p + 1;
    A.need_exact = (u32*)b_ccount.p + 2;
    A.race_keys = (u64*)b_rkeys[0].p;
    A.race_vals = (u32*)b_rvals[0].p;
    A.races = (RaceOut*)b_races.p;
    A.race_cap = race_cap;
    A.cross_list = (u32*)b_cross.p;
    A.tile_flags = (u8*)b_tflags.p;
    A.part = b_part.p;
    A.carry = b_carry.p;
    A.owner = (u32*)b_owner.p;
    A.slots = (Slot*)b_slots.p;
    A.index_base = index_base;
    A.tstart = (const u32*)b_tstart.p;
    A.work = (u32*)b_work.p;
    A.work_count = (u32*)b_ccount.p + 3;
    LAUNCH("tile_starts", 8.0 * m2, launch_tile_starts(A, ctiles, (u32*)b_tstart.p, stream));
    // cheap summaries first; a benign query they cannot decide (>= 2 writers with >= 2 values at one location)
    // makes the whole check rerun with the exact summaries (mode 1 and, for crossing runs, mode 2 can detect it)
    u32 cc[3] = {0, 0, 0};
    for (int pass = 0; pass < 2; pass++) {
      const bool exact = pass == 1;
      cudaMemsetAsync(b_ccount.p, 0, 16, stream);
      LAUNCH(exact ? "conflict_exact" : "conflict", 40.0 * m2, launch_conflict(1, exact, A, ctiles, stream));
      if (!cuda_ok(cudaMemcpyAsync(cc, b_ccount.p, 12, cudaMemcpyDeviceToHost, stream), "counts")) return false;
      if (!sync_check("conflict")) return false;
      if (cc[2] && !exact) continue;
      info.crossing_tiles = cc[1];
      if (cc[1]) {
        LAUNCH("carry", 0.0, launch_carry(exact, A, ctiles, b_carrytmp.p, stream));
        // pieces that start a run first (with position-ordered runs they hold its lowest positions, so the
        // witnesses they find let the other pieces skip), then the rest
        A.phase = 1;
        LAUNCH("conflict_cross", 0.0, launch_conflict(2, exact, A, cc[1], stream));
        A.phase = 2;
        LAUNCH("conflict_cross", 0.0, launch_conflict(2, exact, A, cc[1], stream));
        if (!exact) {
          if (!cuda_ok(cudaMemcpyAsync(cc, b_ccount.p, 12, cudaMemcpyDeviceToHost, stream), "counts")) return false;
          if (!sync_check("crossing")) return false;
          if (cc[2]) continue;
        }
        A.phase = 1;
        LAUNCH("conflict_y", 0.0, launch_conflict(3, exact, A, cc[1], stream));
        A.phase = 2;
        LAUNCH("conflict_y", 0.0, launch_conflict(3, exact, A, cc[1], stream));
        A.phase = 0;
        LAUNCH("cross_emit", 0.0, launch_cross_emit(A, cc[1], stream));
        if (!cuda_ok(cudaMemcpyAsync(cc, b_ccount.p, 12, cudaMemcpyDeviceToHost, stream), "counts")) return false;
        if (!sync_check("crossing")) return false;
      }
      break;
    }
    if (cc[0] <= race_cap) {
      n_races = cc[0];
      return true;
    }
    race_cap = (u32)std::min<u64>((u64)cc[0] + cc[0] / 8 + 1024, 2 * (u64)m2 + 16);
    race_cap_hint = race_cap;
  }
  return fail(SESA_ECUDA, "race list did not fit after retries"), false;
}

// (u64 key, u32 value) pairs sorted stably by the low `bits` key bits (onesweep key/value passes, trivial
// digits skipped); *which = 0 if the result is in (k0, v0), 1 if in (k1, v1)
bool sesa_trace::sort_kv(u64* k0, u32* v0, u64* k1, u32* v1, u32 n, u32 bits, int* which) {
  *which = 0;
  const u32 npass = (bits + RADIX_BITS - 1) / RADIX_BITS;
  if (n == 0 || npass == 0) return true;
  const u32 tiles = sort_tiles(n);
  if (!grow(b_rhist, (size_t)npass * RADIX * 4, "kv hist") || !grow(b_rbase, (size_t)npass * RADIX * 8, "kv base") ||
      !grow(b_lookback, (size_t)tiles * RADIX * 8, "lookback") || !grow(b_ctr, 64 * 4, "counters"))
    return false;
  if (b_lookback.cap != lookback_cleared) {
    cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
    lookback_cleared = b_lookback.cap;
    epoch = 0;
  }
  cudaMemsetAsync(b_rhist.p, 0, (size_t)npass * RADIX * 4, stream);
  cudaMemsetAsync((u32*)b_ctr.p + 32, 0, 32 * 4, stream);
  LAUNCH("kv_hist", 8.0 * n, launch_hist_keys(k0, n, npass, (u32*)b_rhist.p, stream));
  LAUNCH("bin_base", 0.0, launch_bin_base((u32*)b_rhist.p, (u64*)b_rbase.p, npass, stream));
  std::vector<u32> h((size_t)npass * RADIX);
  if (!cuda_ok(cudaMemcpyAsync(h.data(), b_rhist.p, h.size() * 4, cudaMemcpyDeviceToHost, stream), "kv hist") ||
      !sync_check("kv hist"))
    return false;
  u64* k[2] = {k0, k1};
  u32* v[2] = {v0, v1};
  int c = 0;
  for (u32 p = 0; p < npass; p++) {
    if (*std::max_element(h.data() + (size_t)p * RADIX, h.data() + (size_t)(p + 1) * RADIX) == n) continue;
    if (++epoch >= 256) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      epoch = 1;
    }
    LAUNCH("kv_sort", 24.0 * n,
           launch_onesweep(k[c], k[c ^ 1], v[c], v[c ^ 1], n, p * RADIX_BITS, (u64*)b_rbase.p + (size_t)p * RADIX,
                           (u64*)b_lookback.p, (u32*)b_ctr.p + 32 + p, epoch, stream));
    c ^= 1;
  }
  *which = c;
  return true;
}

// step 5b (flags bit 0): benign W/W records, appended to the unsorted race list
// (k_conflict.cu "benign W/W" has the method).  n_races grows by the locations holding a benign pair.
bool sesa_trace::step_benign(const u64* comp, u32 m2, const Rec* rec, u64 index_base, const Rec* rec_entry) {
  if (!(cfg.flags & SESA_FLAG_REPORT_BENIGN) || m2 < 2) return true;
  const KeyLayout& L = layout;
  if (!grow(b_bhead, (size_t)m2 * 4, "benign") || !grow(b_bhscan, (size_t)m2 * 4, "benign") ||
      !grow(b_bwf, (size_t)m2 * 4, "benign") || !grow(b_bwscan, (size_t)m2 * 4, "benign") ||
      !grow(b_bgid, (size_t)m2 * 4, "benign") || !grow(b_temp, scan_u32_temp_bytes(m2), "scan"))
    return false;
  LAUNCH("benign_mark", 16.0 * m2, launch_benign_mark(comp, m2, L, rec, rec_entry, (u32*)b_bhead.p, (u32*)b_bwf.p, stream));
  LAUNCH("scan", 8.0 * m2, launch_scan_exclusive_u32((u32*)b_bhead.p, (u32*)b_bhscan.p, m2, b_temp.p, stream));
  LAUNCH("scan", 8.0 * m2, launch_scan_exclusive_u32((u32*)b_bwf.p, (u32*)b_bwscan.p, m2, b_temp.p, stream));
  u32 tail[4];
  cudaMemcpyAsync(&tail[0], (u32*)b_bwscan.p + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&tail[1], (u32*)b_bwf.p + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&tail[2], (u32*)b_bhscan.p + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&tail[3], (u32*)b_bhead.p + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  if (!sync_check("benign counts")) return false;
  const u32 m3 = tail[0] + tail[1], ngroups = tail[2] + tail[3];
  if (m3 < 2) return true;
  if (!grow(b_bvk[0], (size_t)m3 * 8, "benign") || !grow(b_bvk[1], (size_t)m3 * 8, "benign") ||
      !grow(b_bvi[0], (size_t)m3 * 4, "benign") || !grow(b_bvi[1], (size_t)m3 * 4, "benign") ||
      !grow(b_brh, (size_t)m3 * 4, "benign") || !grow(b_brscan, (size_t)m3 * 4, "benign") ||
      !grow(b_bder, (size_t)m3 * sizeof(Rec), "benign") || !grow(b_bdpos, (size_t)m3 * 4, "benign") ||
      !grow(b_bdj, (size_t)m3 * 4, "benign") || !grow(b_bslot, (size_t)ngroups * 8, "benign") ||
      !grow(b_temp, scan_u32_temp_bytes(m3), "scan"))
    return false;
  LAUNCH("benign_gather", 24.0 * m2,
         launch_benign_gather(comp, m2, L, rec, rec_entry, (const u32*)b_bhead.p, (const u32*)b_bhscan.p, (const u32*)b_bwf.p,
                              (const u32*)b_bwscan.p, (u32*)b_bgid.p, (u64*)b_bvk[0].p, (u32*)b_bvi[0].p, stream));
  // stable LSD passes over the plain-write list -> (location, value, position) order.  Entries of a location
  // are already position-ordered unless global keys carry (block, interval) below the granule (input not in
  // (block, interval) order, lowG > 0): then a position sort comes first.
  int w = 0;
  if (L.lowG != 0) {
    LAUNCH("benign_keys", 12.0 * m3,
           launch_benign_keys(comp, L, rec, rec_entry, (const u32*)b_bvi[0].p, m3, (const u32*)b_bgid.p, 0, (u64*)b_bvk[0].p,
                              stream));
    if (!sort_kv((u64*)b_bvk[0].p, (u32*)b_bvi[0].p, (u64*)b_bvk[1].p, (u32*)b_bvi[1].p, m3, L.pos_bits, &w))
      return false;
    LAUNCH("benign_keys", 40.0 * m3,
           launch_benign_keys(comp, L, rec, rec_entry, (const u32*)b_bvi[w].p, m3, (const u32*)b_bgid.p, 1, (u64*)b_bvk[w].p,
                              stream));
  }
  int w1 = 0;
  if (!sort_kv((u64*)b_bvk[w].p, (u32*)b_bvi[w].p, (u64*)b_bvk[w ^ 1].p, (u32*)b_bvi[w ^ 1].p, m3, 64, &w1))
    return false;
  w ^= w1;
  LAUNCH("benign_keys", 12.0 * m3,
         launch_benign_keys(comp, L, rec, rec_entry, (const u32*)b_bvi[w].p, m3, (const u32*)b_bgid.p, 2, (u64*)b_bvk[w].p,
                            stream));
  u32 gbits = 0;
  while (gbits < 32 && (1ull << gbits) < ngroups) gbits++;
  int w2 = 0;
  if (!sort_kv((u64*)b_bvk[w].p, (u32*)b_bvi[w].p, (u64*)b_bvk[w ^ 1].p, (u32*)b_bvi[w ^ 1].p, m3, gbits, &w2))
    return false;
  const u32* order = (const u32*)(w2 ? b_bvi[w ^ 1].p : b_bvi[w].p);
  LAUNCH("benign_runs", 24.0 * m3,
         launch_benign_runs(comp, L, rec, rec_entry, (const u32*)b_bgid.p, order, m3, (u32*)b_brh.p, stream));
  LAUNCH("scan", 8.0 * m3, launch_scan_exclusive_u32((u32*)b_brh.p, (u32*)b_brscan.p, m3, b_temp.p, stream));
  LAUNCH("benign_derive", 80.0 * m3,
         launch_benign_derive(comp, L, rec, rec_entry, order, (const u32*)b_brh.p, (const u32*)b_brscan.p, m3, (Rec*)b_bder.p,
                              (u32*)b_bdpos.p, (u32*)b_bdj.p, stream));
  if (!sync_check("benign derive")) return false;
  // the derived trace: plain writes with distinct values at (location, value) runs, granularity 1
  if (!child) {
    sesa_config cc = cfg;
    cc.granularity = 1;
    cc.flags = 0;
    if (sesa_trace_create(&cc, &child) != SESA_OK) return fail(SESA_ENOMEM, "benign child handle"), false;
  }
  child->stream = stream;
  child->profiling = false;
  const sesa_status cs = child->check_device((const sesa_access*)b_bder.p, m3, 0);
  launches += child->launches;
  if (cs != SESA_OK) return fail(cs, "benign derived check: %s", child->err.c_str()), false;
  const u32 nc = (u32)child->n_races;
  if (nc == 0) return true;
  // append: keep the n_races records already emitted, grow for nc more
  const u64 need = n_races + nc;
  if (!grow_keep(b_races, need * sizeof(RaceOut), n_races * sizeof(RaceOut), "races") ||
      !grow_keep(b_rkeys[0], need * 8, n_races * 8, "race keys") ||
      !grow_keep(b_rvals[0], need * 4, n_races * 4, "race vals") || !grow(b_rkeys[1], need * 8, "race keys") ||
      !grow(b_rvals[1], need * 4, "race vals") || !grow(b_ccount, 16, "ccount"))
    return false;
  const u32 nr0 = (u32)n_races;
  cudaMemcpyAsync(b_ccount.p, &nr0, 4, cudaMemcpyHostToDevice, stream);
  cudaMemsetAsync(b_bslot.p, 0xFF, (size_t)ngroups * 8, stream);
  ConflictArgs A;
  memset(&A, 0, sizeof A);
  A.keys = comp;
  A.m = m2;
  A.rec = rec;
  A.rec_entry = rec_entry;
  A.L = layout;
  A.race_count = (u32*)b_ccount.p;
  A.race_keys = (u64*)b_rkeys[0].p;
  A.race_vals = (u32*)b_rvals[0].p;
  A.races = (RaceOut*)b_races.p;
  A.race_cap = (u32)need;
  A.index_base = index_base;
  LAUNCH("benign_emit", 0.0,
         launch_benign_min_emit(A, (const RaceOut*)child->b_races_sorted.p, nc, (const u32*)b_bdpos.p,
                                (const u32*)b_bdj.p, (const u32*)b_bgid.p, (unsigned long long*)b_bslot.p, stream));
  u32 total = 0;
  if (!cuda_ok(cudaMemcpyAsync(&total, b_ccount.p, 4, cudaMemcpyDeviceToHost, stream), "benign count") ||
      !sync_check("benign emit"))
    return false;
  n_races = total;
  return true;
}

// step 5' (precise warp model; k_conflict.cu "precise warps" has the method): the
// inter-warp half by the conflict tiles with identity = warp, the intra-warp half pair by pair inside each
// (location, block, interval, warp) group, both folded into per-(run, kind) minimum slots, then emitted
bool sesa_trace::step_warp_model(const u64* comp, u32 m2, const Rec* rec, u64 index_base) {
  const u32 ws = cfg.warp_size;
  // warp size 1: no two threads share a warp, the ordinary check is the model
  conflict_tdiv = ws > 1 ? ws : 0;
  const bool ok = step_conflict(comp, m2, rec, 0, nullptr, index_base);
  conflict_tdiv = 0;
  if (!ok || ws == 1 || m2 < 2) return ok;
  const u32 nA = (u32)n_races;
  const KeyLayout& L = layout;
  if (!grow(b_bhead, (size_t)m2 * 4, "warp") || !grow(b_bhscan, (size_t)m2 * 4, "warp") ||
      !grow(b_bwf, (size_t)m2 * 4, "warp") || !grow(b_bvk[0], (size_t)m2 * 8, "warp") ||
      !grow(b_bvk[1], (size_t)m2 * 8, "warp") || !grow(b_bvi[0], (size_t)m2 * 4, "warp") ||
      !grow(b_bvi[1], (size_t)m2 * 4, "warp") || !grow(b_temp, scan_u32_temp_bytes(m2), "scan"))
    return false;
  u32* head = (u32*)b_bhead.p;
  u32* hscan = (u32*)b_bhscan.p;
  LAUNCH("warp_keys", 40.0 * m2, launch_warp_keys(comp, m2, L, rec, ws, head, (u32*)b_bwf.p, stream));
  LAUNCH("scan", 8.0 * m2, launch_scan_exclusive_u32(head, hscan, m2, b_temp.p, stream));
  u32 tail[2];
  cudaMemcpyAsync(&tail[0], hscan + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&tail[1], head + m2 - 1, 4, cudaMemcpyDeviceToHost, stream);
  if (!sync_check("warp runs")) return false;
  const u32 ngroups = tail[0] + tail[1];
  LAUNCH("warp_key2", 20.0 * m2,
         launch_warp_key2(head, hscan, (const u32*)b_bwf.p, m2, (u64*)b_bvk[0].p, (u32*)b_bvi[0].p, stream));
  u32 gbits = 0;
  while (gbits < 32 && (1ull << gbits) < ngroups) gbits++;
  int w = 0;
  if (!sort_kv((u64*)b_bvk[0].p, (u32*)b_bvi[0].p, (u64*)b_bvk[1].p, (u32*)b_bvi[1].p, m2, 32 + gbits, &w)) return false;
  if (!grow(b_bslot, (size_t)ngroups * 16, "warp slots")) return false;
  unsigned long long* slot = (unsigned long long*)b_bslot.p;
  cudaMemsetAsync(slot, 0xFF, (size_t)ngroups * 16, stream);
  LAUNCH("warp_pairs", 0.0,
         launch_warp_pairs(comp, L, rec, warp_ext, ws, (const u64*)b_bvk[w].p, (const u32*)b_bvi[w].p, m2, slot,
                           stream));
  LAUNCH("warp_fold", 0.0,
         launch_warp_fold((const u64*)b_rkeys[0].p, (const RaceOut*)b_races.p, nA, comp, m2, L, hscan, index_base, slot,
                          stream));
  // re-emit every (run, kind) from its slot
  const u64 need = 2ull * ngroups;
  if (!grow(b_races, need * sizeof(RaceOut), "races") || !grow(b_rkeys[0], need * 8, "race keys") ||
      !grow(b_rkeys[1], need * 8, "race keys") || !grow(b_rvals[0], need * 4, "race vals") ||
      !grow(b_rvals[1], need * 4, "race vals") || !grow(b_ccount, 16, "ccount"))
    return false;
  cudaMemsetAsync(b_ccount.p, 0, 16, stream);
  ConflictArgs A;
  memset(&A, 0, sizeof A);
  A.keys = comp;
  A.m = m2;
  A.rec = rec;
  A.L = L;
  A.race_count = (u32*)b_ccount.p;
  A.race_keys = (u64*)b_rkeys[0].p;
  A.race_vals = (u32*)b_rvals[0].p;
  A.races = (RaceOut*)b_races.p;
  A.race_cap = (u32)need;
  A.index_base = index_base;
  LAUNCH("warp_emit", 0.0, launch_warp_emit(A, head, hscan, slot, stream));
  u32 total = 0;
  if (!cuda_ok(cudaMemcpyAsync(&total, b_ccount.p, 4, cudaMemcpyDeviceToHost, stream), "warp count") ||
      !sync_check("warp emit"))
    return false;
  n_races = total;
  return true;
}

// step 6: canonical order of nr races: sort (location key << 1 | kind, index), permute into `out`
bool sesa_trace::step_race_sort(u32 nr, const RaceOut* races, u64* rkeys0, u32* rvals0, u64* rkeys1, u32* rvals1,
                                RaceOut* out) {
  if (nr == 0) return true;
  const u32 rbits = layout.sort_bits + 2;  // race key = location << 2 | (kind - 1)
  const u32 rpass = (rbits + RADIX_BITS - 1) / RADIX_BITS;
  const u32 rtiles = sort_tiles(nr);
  if (!grow(b_rhist, (size_t)rpass * RADIX * 4, "race hist") || !grow(b_rbase, (size_t)rpass * RADIX * 8, "race base") ||
      !grow(b_lookback, (size_t)rtiles * RADIX * 8, "lookback") || !grow(b_ctr, 64 * 4, "counters"))
    return false;
  if (b_lookback.cap != lookback_cleared) {
    cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
    lookback_cleared = b_lookback.cap;
    epoch = 0;
  }
  cudaMemsetAsync(b_rhist.p, 0, (size_t)rpass * RADIX * 4, stream);
  cudaMemsetAsync((u32*)b_ctr.p + 32, 0, 32 * 4, stream);
  LAUNCH("race_hist", 8.0 * nr, launch_hist_keys(rkeys0, nr, rpass, (u32*)b_rhist.p, stream));
  LAUNCH("bin_base", 0.0, launch_bin_base((u32*)b_rhist.p, (u64*)b_rbase.p, rpass, stream));
  u64* k[2] = {rkeys0, rkeys1};
  u32* v[2] = {rvals0, rvals1};
  int rc = 0;
  for (u32 p = 0; p < rpass; p++) {
    if (++epoch >= 256) {
      cudaMemsetAsync(b_lookback.p, 0, b_lookback.cap, stream);
      epoch = 1;
    }
    LAUNCH("race_sort", 24.0 * nr,
           launch_onesweep(k[rc], k[rc ^ 1], v[rc], v[rc ^ 1], nr, p * RADIX_BITS, (u64*)b_rbase.p + (size_t)p * RADIX,
                           (u64*)b_lookback.p, (u32*)b_ctr.p + 32 + p, epoch, stream));
    rc ^= 1;
  }
  LAUNCH("race_permute", 80.0 * nr, launch_permute_races(races, v[rc], out, nr, stream));
  return true;
}

sesa_status sesa_trace::check_device(const sesa_access* d_rec, u64 n, u64 index_base) {
  begin_check(n);
  if (n == 0) {
    set_oob(d_rec, 0, 0, index_base);
    have_result = true;
    collect_prof();
    return SESA_OK;
  }
  if (!check_records_ptr(d_rec, n)) return status;
  const Rec* rec = reinterpret_cast<const Rec*>(d_rec);
#ifndef SESA_NO_XPART
  {  // C5-like traces: the bucket path with its first partition fused into the extents pass
    bool used = false;
    u64* comp = nullptr;
    u32 m2 = 0;
    if (!try_extents_part(rec, n, index_base, &comp, &m2, &used)) return status;
    if (used) return finish_check(comp, m2, rec, index_base);
    memset(&info, 0, sizeof info);
    info.n_records = n;
  }
#endif
  if (!step_extents(rec, n, true)) return status;
  const Summary& S = h_summary;
  if (S.bad_index != ~0ull) return report_bad(d_rec, S.bad_index, S.bad_index), status;
  set_oob(d_rec, S.oob_count, S.oob_first, index_base);
  const u64 m = S.entries;
  info.n_entries = m;
  info.sorted_input = !S.unsorted;
  if (m >= (1ull << 31)) return fail(SESA_ERANGE, "%llu entries >= 2^31 (ABI v1 limit)", (unsigned long long)m), status;
  if (!make_layout(S, n)) return status;
  info.sort_bits = layout.sort_bits;
  info.pos_bits = layout.pos_bits;
  info.digit_bits = RADIX_BITS;
  const u32 npass = (layout.sort_bits + RADIX_BITS - 1) / RADIX_BITS;
  const bool fused = have_thist && !layout.both && layout.single_space == SP_GLOBAL && layout.lowG == 0 &&
                     S.multi == 0 && m == n && layout.sort_bits <= 32 && fused_supported(npass);
  info.fused_first_pass = fused ? 1 : 0;
  // bucket path: large traces whose granules spread evenly (k_bucket.cu)
  u64 hyb_g0 = 0;
  u32 hyb_nb = 0, hyb_nc = 0;
  if (fused && have_thist2 && !presample_hot && bucket_choose(n, &hyb_g0, &hyb_nb, &hyb_nc)) {
    layout.gminG = hyb_g0;
    layout.gbG = hyb_nb;
    layout.sort_bits = hyb_nb;
    info.sort_bits = hyb_nb;
    info.bucket_path = 1;
    u64* comp = nullptr;
    u32 m2 = 0;
    if (!step_bucket(n, hyb_nc, &comp, &m2)) return status;
    return finish_check(comp, m2, rec, index_base);
  }
  if (status != SESA_OK) return status;
  // Fused path: align gmin down to a multiple of 2^(8 (npass - 1)).  Then every later sort digit of
  // key_hi = g - gmin is a raw granule byte (the top one rotated by a constant), whose histograms the extents
  // pass already took — the fused pass needs no histogram atomics.  Only if the aligned span needs no extra pass.
  hist_from_extents = false;
  if (fused && npass > 1) {
    const u32 D = RADIX_BITS * (npass - 1);
    const u64 G0 = S.gmin[1] & ~((1ull << D) - 1ull);
    const u32 nb = bits_of(S.gmax[1] - G0);
    if ((nb + RADIX_BITS - 1) / RADIX_BITS == npass && nb + layout.pos_bits <= 64) {
      layout.gminG = G0;
      layout.gbG = nb;
      layout.sort_bits = nb;
      info.sort_bits = nb;
      hist_from_extents = true;
    }
  }
  int cur = 0;
  if (fused) {
    // the write bit below the position (KeyLayout::wbit): compaction drops read-only locations
#ifndef SESA_NO_WBIT
    layout.wbit = layout.sort_bits + layout.pos_bits + 1 <= 64 ? 1u : 0u;
#endif
    if (!step_extract_fused(rec, n) || !step_sort(m, &cur, 1, 1)) return status;
  } else {
    // the write bit, unless the key array may still take the bucket path (whose kernels read plain keys)
    const KeyLayout& L = layout;
    const bool bucket_ok = !(m < BUCKET_MIN_N || L.both || (L.single_space == SP_GLOBAL && L.lowG) ||
                             L.sort_bits <= HYB_LO + RADIX_BITS || L.sort_bits > HYB_LO + 2 * RADIX_BITS);
#ifndef SESA_NO_WBIT
    layout.wbit = !bucket_ok && layout.sort_bits + layout.pos_bits + 1 <= 64 ? 1u : 0u;
#endif
    if (!step_extract(rec, n, m, 0, S.multi != 0)) return status;
    bool used = false;
    u64* bcomp = nullptr;
    u32 bm2 = 0;
    if (!try_bucket_keys(m, &bcomp, &bm2, &used)) return status;
    if (used) return finish_check(bcomp, bm2, rec, index_base);
    if (!step_sort(m, &cur)) return status;
  }
  u64* comp = nullptr;
  u32 m2 = 0;
  if (!step_compact(cur, m, &comp, &m2)) return status;
  return finish_check(comp, m2, rec, index_base);
}

// steps 5-6 (shared by the sort + compaction and the bucket paths): conflict tiles, benign regrouping, race sort
sesa_status sesa_trace::finish_check(const u64* comp, u32 m2, const Rec* rec, u64 index_base) {
  if (warp_ext && cfg.lockstep) {
    if (!step_warp_model(comp, m2, rec, index_base)) return status;
  } else {
    if (!step_conflict(comp, m2, rec, 0, nullptr, index_base)) return status;
    if (!step_benign(comp, m2, rec, index_base)) return status;
  }
  const u32 nr = (u32)n_races;
  info.n_races = nr;
  if (!grow(b_races_sorted, (size_t)std::max(nr, 1u) * sizeof(RaceOut), "sorted races")) return status;
  if (!step_race_sort(nr, (RaceOut*)b_races.p, (u64*)b_rkeys[0].p, (u32*)b_rvals[0].p, (u64*)b_rkeys[1].p,
                      (u32*)b_rvals[1].p, (RaceOut*)b_races_sorted.p))
    return status;
  if (!sync_check("race sort")) return status;
  info.launches = launches;
  collect_prof();
  info.n_stats = (u32)stats.size();
  have_result = true;
  return SESA_OK;
}

// ------------------------------------------------------------------------------------------------ launches
// Multi-launch trace (NEXT-4): the launch is part of every location, so the check is the union of the per-launch
// checks; their canonical lists concatenated in launch order are the canonical list ordered by (epoch, ...).
sesa_status sesa_trace::check_launches(const sesa_access* d_rec, u64 n, const u64* offs, u32 nl, u64 index_base) {
  if (!offs || nl == 0) return begin_check(n), fail(SESA_EINVAL, "launch_offsets is NULL or n_launches is 0"), status;
  if (offs[0] != 0 || offs[nl] != n)
    return begin_check(n), fail(SESA_EINVAL, "launch_offsets must start at 0 and end at n"), status;
  for (u32 e = 0; e < nl; e++)
    if (offs[e + 1] < offs[e]) return begin_check(n), fail(SESA_EINVAL, "launch_offsets decrease at %u", e), status;
  u64 total = 0, entries = 0, multi = 0, oob_n = 0, oob_first = ~0ull;
  u32 kernels = 0;
  sesa_access oob_rec;
  memset(&oob_rec, 0, sizeof oob_rec);
  for (u32 e = 0; e < nl; e++) {
    const u64 ne = offs[e + 1] - offs[e];
    const sesa_status st = check_device(ne ? d_rec + offs[e] : d_rec, ne, index_base + offs[e]);
    if (st != SESA_OK) {
      err = "launch " + std::to_string(e) + ": " + err;
      return st;
    }
    entries += info.n_entries, multi += info.n_multi, kernels += launches;
    if (oob.n_oob) {
      if (oob.first_index < oob_first) oob_first = oob.first_index, oob_rec = oob.first;
      oob_n += oob.n_oob;
    }
    const u32 nr = (u32)n_races;
    if (nr) {
      if (!grow_keep(b_lraces, (total + nr) * sizeof(RaceOut), total * sizeof(RaceOut), "launch races")) return status;
      launches++;
      launch_races_set_epoch((const RaceOut*)b_races_sorted.p, nr, e, (RaceOut*)b_lraces.p + total, stream);
      total += nr;
    }
  }
  if (!sync_check("launch races")) return status;
  // the union becomes the handle's result
  if (!grow(b_races_sorted, std::max<u64>(total, 1) * sizeof(RaceOut), "sorted races")) return status;
  if (total && !cuda_ok(cudaMemcpyAsync(b_races_sorted.p, b_lraces.p, total * sizeof(RaceOut), cudaMemcpyDeviceToDevice,
                                        stream), "launch races"))
    return status;
  if (!sync_check("launch races")) return status;
  n_races = total;
  info.n_records = n, info.n_entries = entries, info.n_multi = multi, info.n_races = total, info.launches = kernels;
  memset(&oob, 0, sizeof oob);
  oob.n_oob = oob_n;
  oob.first_index = oob_n ? oob_first : ~0ull;
  oob.first = oob_rec;
  have_oob = true;
  have_result = true;
  return SESA_OK;
}

// ------------------------------------------------------------------------------------------------ flows (NEXT-2)
sesa_status sesa_trace::check_flows(const sesa_flow* d_flows, u64 nf) {
  begin_check(0);
  memset(&flow_info, 0, sizeof flow_info);
  flow_info.n_flows = nf;
  if (nf && !d_flows) return fail(SESA_EINVAL, "d_flows is NULL"), status;
  std::vector<sesa_flow> h(nf);
  if (nf && !cuda_ok(cudaMemcpy(h.data(), d_flows, nf * sizeof(sesa_flow), cudaMemcpyDeviceToHost), "flows D2H"))
    return status;
  u32 bmin = ~0u, bmax = 0, tmax = 0;
  std::vector<u32> ivs;
  for (u64 d = 0; d < nf; d++) {
    const sesa_flow& f = h[d];
    if (f.fkind > 4 || (f.fkind == SESA_F_MODADD && f.fm == 0) || (f.fkind >= SESA_F_SHR && f.fc >= 32) ||
        f.space > 1 || f.rw > 2 || f.size == 0)
      return fail(SESA_EINVAL, "flow %llu invalid", (unsigned long long)d), status;
    ivs.push_back(f.interval);
    if (f.block_lo >= f.block_hi) continue;
    bmin = std::min(bmin, f.block_lo);
    bmax = std::max(bmax, f.block_hi);
    tmax = std::max(tmax, f.nthreads);
  }
  if (nf == 0 || bmin >= bmax || tmax == 0) return check_device(nullptr, 0, 0);
  std::sort(ivs.begin(), ivs.end());
  ivs.erase(std::unique(ivs.begin(), ivs.end()), ivs.end());
  const u32 niv = (u32)ivs.size();
  std::vector<u32> ivoff(niv + 1, 0), idx;
  for (u32 q = 0; q < niv; q++) {
    for (u64 d = 0; d < nf; d++)
      if (h[d].interval == ivs[q]) idx.push_back((u32)d);
    ivoff[q + 1] = (u32)idx.size();
  }
  const u64 ncell = (u64)(bmax - bmin) * niv * tmax;
  if (!grow(b_eoff, (niv + 1 + idx.size()) * 4, "flow csr") || !grow(b_franges, flow_range_bytes((u32)nf), "ranges") ||
      !grow(b_fkeep, nf * 4, "keep") || !grow(b_ecnt, ncell * 4, "cell counts") || !grow(b_ecell, ncell * 4, "cells") ||
      !grow(b_fcnt2, ncell * 4, "cell counts") || !grow(b_foff2, ncell * 4, "cells") ||
      !grow(b_temp, scan_u32_temp_bytes(ncell), "scan"))
    return status;
  u32* d_ivoff = (u32*)b_eoff.p;
  u32* d_idx = d_ivoff + niv + 1;
  cudaMemcpyAsync(d_ivoff, ivoff.data(), ivoff.size() * 4, cudaMemcpyHostToDevice, stream);
  cudaMemcpyAsync(d_idx, idx.data(), idx.size() * 4, cudaMemcpyHostToDevice, stream);
  // (1) the descriptor-pair decisions
  LAUNCH("flow_pairs", 0.0, launch_flow_ranges(d_flows, (u32)nf, (u32)__builtin_ctz(cfg.granularity), b_franges.p,
                                               (u32*)b_fkeep.p, stream));
  std::vector<u32> keep(nf);
  if (!cuda_ok(cudaMemcpyAsync(keep.data(), b_fkeep.p, nf * 4, cudaMemcpyDeviceToHost, stream), "keep")) return status;
  // (2) canonical offsets of the full expansion and of the undecided descriptors' instances
  LAUNCH("flow_count", 8.0 * ncell,
         launch_flow_count_sel(d_flows, d_ivoff, d_idx, niv, bmin, ncell, tmax, (const u32*)b_fkeep.p, (u32*)b_ecnt.p,
                               (u32*)b_fcnt2.p, stream));
  LAUNCH("scan", 8.0 * ncell, launch_scan_exclusive_u32((u32*)b_ecnt.p, (u32*)b_ecell.p, ncell, b_temp.p, stream));
  LAUNCH("scan", 8.0 * ncell, launch_scan_exclusive_u32((u32*)b_fcnt2.p, (u32*)b_foff2.p, ncell, b_temp.p, stream));
  u32 last[4];
  cudaMemcpyAsync(&last[0], (u32*)b_ecell.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&last[1], (u32*)b_ecnt.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&last[2], (u32*)b_foff2.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&last[3], (u32*)b_fcnt2.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  if (!sync_check("flow counts")) return status;
  u64 bound = 0;  // the u32 scans wrap past 2^32: refuse before (sum of per-flow maxima)
  for (u64 d = 0; d < nf; d++)
    if (h[d].block_lo < h[d].block_hi)
      bound += (u64)(h[d].block_hi - h[d].block_lo) * std::min<u64>(h[d].nthreads, h[d].phi > h[d].plo ? h[d].phi - h[d].plo : 0) * h[d].count;
  if (bound >= (1ull << 31)) return fail(SESA_ERANGE, "the flows may describe >= 2^31 records"), status;
  const u64 total = (u64)last[0] + last[1], kept = (u64)last[2] + last[3];
  u64 nkept_flows = 0;
  for (u64 d = 0; d < nf; d++) nkept_flows += keep[d] ? 1 : 0;
  // (3) instantiate the undecided descriptors only, with their canonical indices; (4) check them
  if (!grow(b_frec, std::max<u64>(kept, 1) * sizeof(Rec), "flow records") || !grow(b_forig, std::max<u64>(kept, 1) * 4, "orig"))
    return status;
  if (kept)
    LAUNCH("flow_write", 36.0 * kept,
           launch_flow_write_sel(d_flows, d_ivoff, d_idx, niv, bmin, ncell, tmax, (const u32*)b_fkeep.p,
                                 (const u32*)b_ecell.p, (const u32*)b_foff2.p, (Rec*)b_frec.p, (u32*)b_forig.p, stream));
  if (!sync_check("flow write")) return status;
  const u32 k0 = launches;
  const sesa_status st = check_device((const sesa_access*)b_frec.p, kept, 0);
  if (st != SESA_OK) return st;
  launches += k0;
  if (n_races) {
    launches++;
    launch_race_remap((RaceOut*)b_races_sorted.p, (u32)n_races, (const u32*)b_forig.p, stream);
  }
  if (oob.n_oob) {
    u32 o = 0;
    cudaMemcpy(&o, (const u32*)b_forig.p + oob.first_index, 4, cudaMemcpyDeviceToHost);
    oob.first_index = o;
  }
  if (!sync_check("race remap")) return status;
  info.launches = launches;
  info.n_records = total;
  flow_info.n_flows_checked = nkept_flows;
  flow_info.n_records = total;
  flow_info.n_records_checked = kept;
  return SESA_OK;
}

// ------------------------------------------------------------------------------------------------ expand
sesa_status sesa_trace::expand(const sesa_flow* d_flows, u64 nf, sesa_access* d_out, u64 cap, u64* n_out) {
  status = SESA_OK;
  err.clear();
  launches = 0;
  prof.clear();
  ev_used = 0;
  if (!n_out) return fail(SESA_EINVAL, "n_out is NULL"), status;
  *n_out = 0;
  if (nf == 0) return SESA_OK;
  if (!d_flows) return fail(SESA_EINVAL, "d_flows is NULL"), status;
  std::vector<sesa_flow> h(nf);
  if (!cuda_ok(cudaMemcpy(h.data(), d_flows, nf * sizeof(sesa_flow), cudaMemcpyDeviceToHost), "flows D2H")) return status;
  u32 bmin = ~0u, bmax = 0, tmax = 0;
  std::vector<u32> ivs;
  for (u64 d = 0; d < nf; d++) {
    const sesa_flow& f = h[d];
    if (f.fkind > 4 || (f.fkind == SESA_F_MODADD && f.fm == 0) || (f.fkind >= SESA_F_SHR && f.fc >= 32))
      return fail(SESA_EINVAL, "flow %llu: bad f (fkind=%u fc=%u fm=%u)", (unsigned long long)d, f.fkind, f.fc, f.fm),
             status;
    if (f.space > 1 || f.rw > 2 || f.size == 0)
      return fail(SESA_EINVAL, "flow %llu: bad access (space=%u rw=%u size=%u)", (unsigned long long)d, f.space, f.rw,
                  f.size),
             status;
    ivs.push_back(f.interval);
    if (f.block_lo >= f.block_hi) continue;
    bmin = std::min(bmin, f.block_lo);
    bmax = std::max(bmax, f.block_hi);
    tmax = std::max(tmax, f.nthreads);
  }
  if (bmin >= bmax || tmax == 0) return SESA_OK;
  std::sort(ivs.begin(), ivs.end());
  ivs.erase(std::unique(ivs.begin(), ivs.end()), ivs.end());
  const u32 niv = (u32)ivs.size();
  std::vector<u32> ivoff(niv + 1, 0), idx;
  for (u32 q = 0; q < niv; q++) {
    u64 csum = 0;
    for (u64 d = 0; d < nf; d++)
      if (h[d].interval == ivs[q]) idx.push_back((u32)d), csum += h[d].count;
    ivoff[q + 1] = (u32)idx.size();
    if (csum >= (1ull << 32)) return fail(SESA_ERANGE, "flow counts of one interval exceed 2^32"), status;
  }
  const u64 ncell = (u64)(bmax - bmin) * niv * tmax;
  if (!grow(b_eoff, (niv + 1 + idx.size()) * 4, "flow csr") || !grow(b_ecnt, ncell * 4, "cell counts") ||
      !grow(b_ecell, ncell * 4, "cell offsets") || !grow(b_temp, scan_u32_temp_bytes(ncell), "scan"))
    return status;
  u32* d_ivoff = (u32*)b_eoff.p;
  u32* d_idx = d_ivoff + niv + 1;
  cudaMemcpyAsync(d_ivoff, ivoff.data(), ivoff.size() * 4, cudaMemcpyHostToDevice, stream);
  cudaMemcpyAsync(d_idx, idx.data(), idx.size() * 4, cudaMemcpyHostToDevice, stream);
  LAUNCH("flow_count", 4.0 * ncell, launch_flow_count2(d_flows, d_ivoff, d_idx, niv, bmin, ncell, tmax, (u32*)b_ecnt.p, stream));
  // total = sum of cell counts: scan then last offset + last count (u64 check for overflow below)
  LAUNCH("scan", 8.0 * ncell, launch_scan_exclusive_u32((u32*)b_ecnt.p, (u32*)b_ecell.p, ncell, b_temp.p, stream));
  u32 last[2];
  cudaMemcpyAsync(&last[0], (u32*)b_ecell.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  cudaMemcpyAsync(&last[1], (u32*)b_ecnt.p + ncell - 1, 4, cudaMemcpyDeviceToHost, stream);
  if (!sync_check("flow count")) return status;
  const u64 total = (u64)last[0] + last[1];
  // overflow guard: the u32 scan wraps past 2^32; recount on the host side of the bound (sum of per-flow maxima)
  u64 bound = 0;
  for (u64 d = 0; d < nf; d++)
    if (h[d].block_lo < h[d].block_hi)
      bound += (u64)(h[d].block_hi - h[d].block_lo) * std::min<u64>(h[d].nthreads, h[d].phi > h[d].plo ? h[d].phi - h[d].plo : 0) * h[d].count;
  if (bound >= (1ull << 32) && total < bound / 2)
    return fail(SESA_ERANGE, "expansion may exceed 2^32 records"), status;
  *n_out = total;
  if (total > cap) return fail(SESA_ETRUNC, "expansion produces %llu records > cap %llu", (unsigned long long)total,
                               (unsigned long long)cap),
                      status;
  if (!d_out) return fail(SESA_EINVAL, "d_out is NULL"), status;
  LAUNCH("flow_write", 32.0 * total,
         launch_flow_write2(d_flows, d_ivoff, d_idx, niv, bmin, ncell, tmax, (u32*)b_ecell.p, (Rec*)d_out, stream));
  if (!sync_check("flow write")) return status;
  collect_prof();
  return SESA_OK;
}

// ------------------------------------------------------------------------------------------------ C ABI
extern "C" {

int sesa_abi_version(void) { return SESA_ABI_VERSION; }

const char* sesa_status_str(sesa_status s) {
  switch (s) {
    case SESA_OK: return "SESA_OK";
    case SESA_EINVAL: return "SESA_EINVAL";
    case SESA_ERANGE: return "SESA_ERANGE";
    case SESA_ENOMEM: return "SESA_ENOMEM";
    case SESA_ECUDA: return "SESA_ECUDA";
    case SESA_ENCCL: return "SESA_ENCCL";
    case SESA_ESTATE: return "SESA_ESTATE";
    case SESA_ETRUNC: return "SESA_ETRUNC";
  }
  return "SESA_?";
}

static sesa_status check_cfg(const sesa_config* c) {
  if (!c) return SESA_EINVAL;
  if (c->warp_size < 1 || c->lockstep > 1 || c->granularity < 1 || c->granularity > 4096 ||
      (c->granularity & (c->granularity - 1)) || (c->flags & ~(uint32_t)SESA_FLAG_REPORT_BENIGN) != 0)
    return SESA_EINVAL;
  return SESA_OK;
}

sesa_status sesa_trace_create(const sesa_config* cfg, sesa_trace** out) {
  if (!out) return SESA_EINVAL;
  *out = nullptr;
  if (check_cfg(cfg) != SESA_OK) return SESA_EINVAL;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return SESA_ECUDA;
  }
  sesa_trace* t = new (std::nothrow) sesa_trace();
  if (!t) return SESA_ENOMEM;
  t->cfg = *cfg;
  t->device = dev;
  t->num_sms = sesa::dev_sm_count();
  *out = t;
  return SESA_OK;
}

sesa_status sesa_race_check(sesa_trace* t, const sesa_access* d_records, uint64_t n, uint64_t index_base,
                            void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  if (t->dist) return t->check_dist(d_records, n, index_base);
  return t->check_device(d_records, n, index_base);
}

sesa_status sesa_race_check_host(sesa_trace* t, const sesa_access* h_records, uint64_t n, uint64_t index_base,
                                 void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  t->status = SESA_OK;
  t->have_result = false;
  if (n == 0) return sesa_race_check(t, nullptr, 0, index_base, cuda_stream);
  if (!h_records) return t->fail(SESA_EINVAL, "h_records is NULL"), t->status;
  if (!t->grow(t->b_hrec, n * sizeof(sesa_access), "record copy")) return t->status;
  const size_t bytes = n * sizeof(sesa_access);
  cudaPointerAttributes pa;
  const bool pinned = cudaPointerGetAttributes(&pa, h_records) == cudaSuccess && pa.type == cudaMemoryTypeHost;
  cudaGetLastError();
  if (pinned) {  // page-locked: one DMA
    if (!t->cuda_ok(cudaMemcpyAsync(t->b_hrec.p, h_records, bytes, cudaMemcpyHostToDevice, t->stream), "records H2D"))
      return t->status;
  } else {
    // pageable: chunked through two page-locked staging buffers; the host copy of chunk i + 1 overlaps the DMA
    // of chunk i
    const size_t CH = 64ull << 20;
    if (!t->h_pinned && !t->cuda_ok(cudaMallocHost(&t->h_pinned, 2 * CH), "pinned staging")) return t->status;
    cudaEvent_t ev[2];
    for (auto& e : ev) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    bool ok = true;
    for (size_t off = 0, i = 0; off < bytes && ok; off += CH, i++) {
      const size_t len = std::min(CH, bytes - off);
      char* stage = (char*)t->h_pinned + (i & 1) * CH;
      if (i >= 2) cudaEventSynchronize(ev[i & 1]);  // its previous DMA has finished
      memcpy(stage, (const char*)h_records + off, len);
      ok = t->cuda_ok(cudaMemcpyAsync((char*)t->b_hrec.p + off, stage, len, cudaMemcpyHostToDevice, t->stream),
                      "records H2D") &&
           t->cuda_ok(cudaEventRecord(ev[i & 1], t->stream), "records H2D");
    }
    for (auto& e : ev) cudaEventDestroy(e);  // (destroy after pending records complete is allowed)
    if (!ok) return t->status;
  }
  return sesa_race_check(t, (const sesa_access*)t->b_hrec.p, n, index_base, cuda_stream);
}

sesa_status sesa_race_check_launches(sesa_trace* t, const sesa_access* d_records, uint64_t n,
                                     const uint64_t* launch_offsets, uint32_t n_launches, uint64_t index_base,
                                     void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  if (t->dist) return t->begin_check(n), t->fail(SESA_EINVAL, "multi-launch checks need a single-GPU handle"), SESA_EINVAL;
  return t->check_launches(d_records, n, launch_offsets, n_launches, index_base);
}

sesa_status sesa_race_check_warp(sesa_trace* t, const sesa_access* d_records, const sesa_access_ext* d_ext,
                                 uint64_t n, uint64_t index_base, void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  if (t->dist) return t->begin_check(n), t->fail(SESA_EINVAL, "the precise warp model needs a single-GPU handle"), SESA_EINVAL;
  if (t->cfg.flags & SESA_FLAG_REPORT_BENIGN)
    return t->begin_check(n), t->fail(SESA_EINVAL, "benign reporting is not defined for the precise warp model"),
           SESA_EINVAL;
  if (n && !d_ext) return t->begin_check(n), t->fail(SESA_EINVAL, "d_ext is NULL"), SESA_EINVAL;
  t->warp_ext = d_ext;
  const sesa_status st = t->check_device(d_records, n, index_base);
  t->warp_ext = nullptr;
  return st;
}

sesa_status sesa_race_check_flows(sesa_trace* t, const sesa_flow* d_flows, uint64_t n_flows, void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  if (t->dist) return t->begin_check(0), t->fail(SESA_EINVAL, "descriptor checks need a single-GPU handle"), SESA_EINVAL;
  return t->check_flows(d_flows, n_flows);
}

sesa_status sesa_flow_check_get(const sesa_trace* t, sesa_flow_check_info* out) {
  if (!t || !out) return SESA_EINVAL;
  if (!t->have_result) return SESA_ESTATE;
  *out = t->flow_info;
  return SESA_OK;
}

sesa_status sesa_races_get(sesa_trace* t, sesa_race* host_out, uint64_t cap, uint64_t* n_races) {
  if (!t || !n_races) return SESA_EINVAL;
  if (!t->have_result) return SESA_ESTATE;
  const u64 nr = t->dist && t->rank != 0 ? 0 : t->n_races;
  *n_races = nr;
  if (cap == 0 || nr == 0) return SESA_OK;
  if (!host_out) return SESA_EINVAL;
  const u64 k = std::min<u64>(cap, nr);
  const void* src = t->dist ? t->b_dist_races.p : t->b_races_sorted.p;
  if (cudaMemcpy(host_out, src, k * sizeof(sesa_race), cudaMemcpyDeviceToHost) != cudaSuccess) {
    cudaGetLastError();
    return SESA_ECUDA;
  }
  return k < nr ? SESA_ETRUNC : SESA_OK;
}

sesa_status sesa_races_device(sesa_trace* t, const sesa_race** d_races, uint64_t* n_races) {
  if (!t || !d_races || !n_races) return SESA_EINVAL;
  if (!t->have_result) return SESA_ESTATE;
  *n_races = t->dist && t->rank != 0 ? 0 : t->n_races;
  *d_races = (const sesa_race*)(t->dist ? t->b_dist_races.p : t->b_races_sorted.p);
  return SESA_OK;
}

sesa_status sesa_expand(sesa_trace* t, const sesa_flow* d_flows, uint64_t n_flows, sesa_access* d_out, uint64_t cap,
                        uint64_t* n_out, void* cuda_stream) {
  if (!t) return SESA_EINVAL;
  t->stream = (cudaStream_t)cuda_stream;
  return t->expand(d_flows, n_flows, d_out, cap, n_out);
}

sesa_status sesa_trace_set_profiling(sesa_trace* t, int enable) {
  if (!t) return SESA_EINVAL;
  t->profiling = enable != 0;
  return SESA_OK;
}

sesa_status sesa_trace_info(const sesa_trace* t, sesa_check_info* out) {
  if (!t || !out) return SESA_EINVAL;
  *out = t->info;
  return SESA_OK;
}

sesa_status sesa_trace_set_regions(sesa_trace* t, const sesa_region* regions, uint32_t n) {
  if (!t || (n && !regions)) return SESA_EINVAL;
  if (n > (uint32_t)MAX_REGIONS) return t->fail(SESA_EINVAL, "%u regions > %d", n, MAX_REGIONS), SESA_EINVAL;
  std::vector<sesa_region> v(regions, regions + n);
  for (uint32_t i = 0; i < n; i++) {
    const sesa_region& r = v[i];
    if (r.space > 1 || r.size == 0 || r.reserved != 0 || r.base + r.size < r.base)
      return t->fail(SESA_EINVAL, "region %u invalid (space=%u size=%llu)", i, r.space, (unsigned long long)r.size),
             SESA_EINVAL;
  }
  std::sort(v.begin(), v.end(), [](const sesa_region& a, const sesa_region& b) {
    return a.space != b.space ? a.space < b.space : a.base < b.base;
  });
  uint32_t nsh = 0;
  for (uint32_t i = 0; i < n; i++) {
    if (v[i].space == SP_SHARED) nsh++;
    if (i && v[i].space == v[i - 1].space && v[i - 1].base + v[i - 1].size > v[i].base)
      return t->fail(SESA_EINVAL, "regions overlap (space %u, base 0x%llx)", v[i].space,
                     (unsigned long long)v[i].base), SESA_EINVAL;
  }
  std::vector<Region> dev(n);
  for (uint32_t i = 0; i < n; i++) dev[i].base = v[i].base, dev[i].end = v[i].base + v[i].size;
  if (n) {
    if (!t->grow(t->b_regions, n * sizeof(Region), "regions")) return t->status;
    if (!t->cuda_ok(cudaMemcpy(t->b_regions.p, dev.data(), n * sizeof(Region), cudaMemcpyHostToDevice), "regions"))
      return t->status;
  }
  t->n_regions = n;
  t->n_regions_shared = nsh;
  return SESA_OK;
}

sesa_status sesa_oob_get(const sesa_trace* t, sesa_oob_report* out) {
  if (!t || !out) return SESA_EINVAL;
  if (!t->have_result || !t->have_oob) return SESA_ESTATE;
  *out = t->oob;
  return SESA_OK;
}

sesa_status sesa_trace_kernel_stats(const sesa_trace* t, sesa_kernel_stat* out, uint32_t cap, uint32_t* n_out) {
  if (!t || !n_out) return SESA_EINVAL;
  *n_out = (u32)t->stats.size();
  for (u32 i = 0; i < std::min<u32>(cap, (u32)t->stats.size()); i++) out[i] = t->stats[i];
  return SESA_OK;
}

void sesa_trace_destroy(sesa_trace* t) {
  if (!t) return;
  t->destroy_dist();
  if (t->child) sesa_trace_destroy(t->child), t->child = nullptr;
  t->free_all();
  delete t;
}

const char* sesa_last_error(const sesa_trace* t) { return t ? t->err.c_str() : ""; }

}  // extern "C"
