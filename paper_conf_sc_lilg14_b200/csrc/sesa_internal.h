// sesa_internal.h — the opaque handle behind include/sesa.h (host side).
#pragma once
#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "../../include/sesa.h"
#include "kernels.cuh"

struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
};

struct ProfRec {
  std::string name;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  double bytes = 0;
};

struct DistState;  // dist.cu

struct sesa_trace {
  sesa_config cfg{};
  int device = 0;
  int num_sms = 148;
  cudaStream_t stream = nullptr;
  sesa_status status = SESA_OK;
  std::string err;
  bool have_result = false;
  uint64_t n_races = 0;
  uint32_t tile_shift = 0;
  uint64_t race_cap_hint = 0;
  uint32_t epoch = 0;
  size_t lookback_cleared = 0;
  sesa::KeyLayout layout{};
  sesa::Summary h_summary{};
  sesa_check_info info{};

  // device buffers (grow-only, freed by destroy)
  DevBuf b_summary, b_keys[2], b_hist, b_binbase, b_lookback, b_ctr, b_cnt, b_off, b_temp;
  DevBuf b_tflags, b_part, b_carry, b_owner, b_slots, b_cross, b_ccount, b_carrytmp, b_tstart, b_work;
  DevBuf b_races, b_rkeys[2], b_rvals[2], b_races_sorted, b_rhist, b_rbase;
  DevBuf b_eoff, b_ecnt, b_ecell, b_hrec, b_dist_races, b_ctmp, b_ctotal, b_thist, b_ftmp, b_thist2, b_btmp2;
  DevBuf b_wbits;   // per-record write bits from the extents pass (KeyLayout::wbit)
  DevBuf b_xtmp, b_xsmall;  // fused extents + first partition: record sample; region fills, overflow, tile prefix
  DevBuf b_lraces;  // multi-launch checks: the races of the launches checked so far
  DevBuf b_franges, b_fkeep, b_fcnt2, b_foff2, b_frec, b_forig;  // descriptor-level check (NEXT-2)
  sesa_flow_check_info flow_info{};
  const void* warp_ext = nullptr;  // precise warp model: the {pc, div} extension of the records being checked
  uint32_t conflict_tdiv = 0;      // > 1: conflict tiles with identity = thread / tdiv, lockstep off
  bool presample_hot = false;  // this check's record sample found a hot chunk: the bucket path cannot pay
  bool have_thist2 = false;  // extents also wrote the per-tile histograms of the bucket path's first digit
  bool have_thist = false;
  bool hist_from_extents = false;  // fused path: later-digit histograms from the extents' raw granule bytes  // extents wrote per-tile raw digit histograms (fused first pass possible)
  // out-of-bound check (NEXT-1): registered regions (sorted by space, base) and the last report
  DevBuf b_regions;
  // benign W/W reporting (flags bit 0): regrouped plain writes and the derived trace checked by `child`
  DevBuf b_bhead, b_bhscan, b_bwf, b_bwscan, b_bgid, b_bvk[2], b_bvi[2], b_brh, b_brscan, b_bder, b_bdpos, b_bdj,
      b_bslot, b_btmp;
  sesa_trace* child = nullptr;
  uint32_t n_regions = 0, n_regions_shared = 0;
  sesa_oob_report oob{};
  bool have_oob = false;
  DevBuf b_dist[8];
  void* h_pinned = nullptr;

  std::vector<DevBuf*> all_bufs() {
    std::vector<DevBuf*> v = {&b_summary, &b_hist, &b_binbase, &b_lookback, &b_ctr, &b_cnt, &b_off, &b_temp,
                              &b_tflags, &b_part, &b_carry, &b_owner, &b_slots, &b_cross, &b_ccount, &b_carrytmp, &b_tstart, &b_work,
                              &b_races, &b_races_sorted, &b_rhist, &b_rbase, &b_eoff, &b_ecnt, &b_ecell,
                              &b_hrec, &b_dist_races, &b_ctmp, &b_ctotal, &b_thist, &b_ftmp, &b_thist2, &b_btmp2, &b_lraces, &b_franges, &b_fkeep, &b_fcnt2,
                              &b_foff2, &b_frec, &b_forig, &b_regions,
                              &b_bhead, &b_bhscan, &b_bwf, &b_bwscan, &b_bgid, &b_bvk[0], &b_bvk[1], &b_bvi[0],
                              &b_bvi[1], &b_brh, &b_brscan, &b_bder, &b_bdpos, &b_bdj, &b_bslot, &b_btmp};
    for (auto& b : b_keys) v.push_back(&b);
    for (auto& b : b_rkeys) v.push_back(&b);
    for (auto& b : b_rvals) v.push_back(&b);
    for (auto& b : b_dist) v.push_back(&b);
    return v;
  }

  // profiling
  bool profiling = false;
  uint32_t launches = 0;
  std::vector<ProfRec> prof;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  std::vector<sesa_kernel_stat> stats;
  std::string prof_last;

  // distributed
  bool dist = false;
  int rank = 0, world = 1;
  DistState* ds = nullptr;

  void fail(sesa_status s, const char* fmt, ...);
  bool cuda_ok(cudaError_t e, const char* what);
  bool grow(DevBuf& b, size_t bytes, const char* what);
  bool grow_keep(DevBuf& b, size_t bytes, size_t used, const char* what);  // preserves the first `used` bytes
  bool sync_check(const char* what);
  void free_all();
  void launch_begin(const char* name);
  void launch_end(double bytes);
  cudaEvent_t next_event();
  void collect_prof();
  bool make_layout(const sesa::Summary& S, uint64_t n);
  sesa_status check_device(const sesa_access* d_rec, uint64_t n, uint64_t index_base);
  sesa_status check_launches(const sesa_access* d_rec, uint64_t n, const uint64_t* offs, uint32_t nl,
                             uint64_t index_base);
  bool step_warp_model(const uint64_t* comp, uint32_t m2, const sesa::Rec* rec, uint64_t index_base);
  sesa_status finish_check(const uint64_t* comp, uint32_t m2, const sesa::Rec* rec, uint64_t index_base);
  // pipeline steps (shared by the single-GPU and the distributed check)
  void begin_check(uint64_t n);
  bool check_records_ptr(const sesa_access* d_rec, uint64_t n);
  bool step_extents(const sesa::Rec* rec, uint64_t n, bool tile_hist = false, uint32_t* gran_out = nullptr);
  bool report_bad(const sesa_access* d_rec, uint64_t local_bad, uint64_t global_bad);
  void set_oob(const sesa_access* d_rec, uint64_t count, uint64_t local_first, uint64_t index_base);
  bool step_extract(const sesa::Rec* rec, uint64_t n, uint64_t m, uint64_t pos_base, bool multi);
  bool step_hist(uint64_t m);
  bool step_extract_fused(const sesa::Rec* rec, uint64_t n);
  bool bucket_choose(uint64_t n, uint64_t* gmin_aligned, uint32_t* nbits, uint32_t* nchunks);
  bool step_bucket(uint64_t n, uint32_t nchunks, uint64_t** comp, uint32_t* m2);
  bool try_bucket_keys(uint64_t m, uint64_t** comp, uint32_t* m2, bool* used);
  bool try_extents_part(const sesa::Rec* rec, uint64_t n, uint64_t index_base, uint64_t** comp, uint32_t* m2,
                        bool* used);
  bool step_sort(uint64_t m, int* cur_out, uint32_t first_pass = 0, int cur0 = 0);
  bool step_compact(int cur, uint64_t m, uint64_t** comp, uint32_t* m2);
  bool step_conflict(const uint64_t* comp, uint32_t m2, const sesa::Rec* rec, uint32_t rec_pos_base,
                     const sesa::Rec* rec_entry, uint64_t index_base);
  bool sort_kv(uint64_t* k0, uint32_t* v0, uint64_t* k1, uint32_t* v1, uint32_t n, uint32_t bits, int* which);
  bool step_benign(const uint64_t* comp, uint32_t m2, const sesa::Rec* rec, uint64_t index_base,
                   const sesa::Rec* rec_entry = nullptr);
  bool step_race_sort(uint32_t nr, const sesa::RaceOut* races, uint64_t* rk0, uint32_t* rv0, uint64_t* rk1,
                      uint32_t* rv1, sesa::RaceOut* out);
  sesa_status check_flows(const sesa_flow* d_flows, uint64_t nf);
  sesa_status expand(const sesa_flow* d_flows, uint64_t nf, sesa_access* d_out, uint64_t cap, uint64_t* n_out);
  sesa_status check_dist(const sesa_access* d_rec, uint64_t n, uint64_t index_base);
  void destroy_dist();
};
