// kernels.cuh — launcher declarations of the sm_100a pipeline kernels.
#pragma once
#include "common.cuh"

namespace sesa {

constexpr int RADIX_BITS = 8;  // onesweep digit width (8-bit digits, 256 bins per pass)
constexpr int RADIX = 1 << RADIX_BITS;
// fused key extract + first sort pass (k_fused.cu): tiles of 256 threads x FUSED_ITEMS records (stable variant,
// C3/C4: 16 items at 3 CTAs/SM — C3 5.88 -> 5.81 ms, C4 extract 2.10 -> 2.01 ms against 24 at 2; 20 at 3 between)
// (unstable variant, C5: 24 items at 2 CTAs/SM 3.75 ms; at 3 CTAs/SM 3.72; 16 items at 3-4 CTAs/SM 4.8-5.0;
// 32 items 3.65 but the extents pass's per-tile histograms slow it by 0.18 ms)
#ifndef FUSED_ITEMS_
#define FUSED_ITEMS_ 16
#endif
#ifndef FUSED_MINB_
#define FUSED_MINB_ 3
#endif
constexpr int FUSED_THREADS = 256, FUSED_ITEMS = FUSED_ITEMS_, FUSED_MINB = FUSED_MINB_, FUSED_TILE = FUSED_THREADS * FUSED_ITEMS;
constexpr int FUSED_UMINB = 2;  // CTAs per SM of the bucket path's unstable variant

// onesweep tile: 256 threads x 16 keys (warp-striped); one lookback word per (tile, bin)
constexpr int SORT_THREADS = 256;
constexpr int SORT_ITEMS = 16;
constexpr int SORT_TILE = SORT_THREADS * SORT_ITEMS;

// conflict tile: 256 threads x 6 entries (blocked; 1536-entry capacity, 3 CTAs/SM — measured against 4, 5, 7, 8:
// C2 3.01 -> 2.62, C3 18.4 -> 16.1, C4 65.1 -> 55.7 ms from 8; 7 re-measured on the final tree: C3 7.76 -> 9.37,
// C4 41.0 -> 45.3 ms, 2 CTAs/SM; 5 with mode 1 at 4 CTAs/SM / 64 registers: C3 7.76 -> 8.91, C4 41.0 -> 44.5 ms)
constexpr int CT_THREADS = 256;
constexpr int CT_ITEMS = 6;
constexpr int CT_TILE = CT_THREADS * CT_ITEMS;

// k_extract.cu
// tile_hist (optional, [ceil(n / FUSED_TILE)][RADIX]): per-tile histograms of (addr >> log2G) & 255 (k_fused.cu)
// regs (optional, device, nreg <= MAX_REGIONS): sorted by (space, base), the first nreg_shared are SHARED
// gout (optional, n x u32): low 32 bits of the granule index addr >> log2G of every record (fused-pass input)
// tile_hist2 (optional, needs tile_hist): per-tile histograms of (addr >> log2G >> HYB_LO) & 255 (k_bucket.cu)
// wout (optional, needs tile_hist, ceil(n / 32) x u32): bit i & 31 of wout[i >> 5] = record i writes (KeyLayout::wbit)
void launch_extents(const Rec* rec, u64 n, u32 log2G, Summary* d_sum, u32* tile_hist, const Region* regs, u32 nreg,
                    u32 nreg_shared, int grid, cudaStream_t st, u32* gout = nullptr, u32* tile_hist2 = nullptr,
                    u32* wout = nullptr);
// extents fused with the bucket path's first partition (k_extract.cu "Extents fused with ...")
struct XPArgs {
  const Rec* rec;
  u32 n, log2G, pos_bits;
  Summary* out;      // initialised like for launch_extents; bhist[3] = raw (g >> 22) & 255 histogram
  u64* kout;         // RADIX regions of cap keys: region d = kout[d * cap, (d + 1) * cap)
  u64 cap;
  u32* gfill;        // [RADIX] zeroed: slots reserved per region (used, sentinel-padded)
  u32* overflow;     // zeroed; 1 if a region would pass cap
};
void launch_extents_part(const XPArgs& A, cudaStream_t st);
// tile of the second partition pass over the regions (k_sort.cu OS_UCFG3)
#ifndef R3_THREADS_
#define R3_THREADS_ 256
#endif
#ifndef R3_ITEMS_
#define R3_ITEMS_ 24
#endif
#ifndef R3_MINB_
#define R3_MINB_ 3
#endif
constexpr u32 PART_TILE_KEYS = R3_THREADS_ * R3_ITEMS_;
// the second partition pass over launch_extents_part's regions: tpr tiles per region (cap is a multiple of
// PART_TILE_KEYS, tpr * PART_TILE_KEYS >= every fill), keys rebased from raw low-30 granule bits by g0
void launch_partition_regions(const u64* kin, u64* kout, u32 tpr, u32 shift, const u64* bin_base, u64* lookback,
                              u32* tile_ctr, u32 epoch, const u32* fill, u64 cap, u32 pos_bits, u32 g0,
                              cudaStream_t st);
u64 extents_part_cap(u64 n);
size_t presample_temp_bytes();
void launch_presample(const Rec* rec, u32 n, u32 log2G, u32 want, void* temp, unsigned long long* h_ext,
                      u32* samples, cudaStream_t st);
void launch_extract_1to1(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, u64* keys, u32* hist, u64 pos_base,
                         int grid, cudaStream_t st);
void launch_entry_count(const Rec* rec, u64 n, u32 log2G, u32* cnt, cudaStream_t st);
void launch_extract_multi(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, const u32* off, u64* keys,
                          u32* hist, u64 pos_base, int grid, cudaStream_t st);

// k_fused.cu — key extract fused with the first sort pass (single global space, (block, interval)-ordered
// input, one granule per record); tile_hist from launch_extents
bool fused_supported(u32 npass);
size_t fused_temp_bytes(u64 n);
// dsh: the digit is key_hi bits [dsh, dsh + 8) (tile_hist then holds the raw (g >> dsh) & 255 histograms and gmin
// is a multiple of 2^dsh)
// pad_kout (bucket path): pad every digit run of the output to a multiple of 32 with ~0 sentinels; *mtot (device)
// = the padded length
void launch_tile_offsets(u64 n, const KeyLayout& L, const u32* tile_hist, void* temp, cudaStream_t st, u32 dsh = 0,
                         u64* pad_kout = nullptr, u32* mtot = nullptr);
// gran: the extents pass's granule indices (gout); rec is not read
// unstable: no stable order within a digit (the bucket path); npass must be 1
void launch_fused_extract_pass0(const u32* gran, u64 n, const KeyLayout& L, u32 npass, void* temp, u64* kout,
                                u32* hist, cudaStream_t st, u32 dsh = 0, bool unstable = false,
                                const u32* wbits = nullptr);  // wbits: extents' wout, needed when L.wbit

constexpr uint64_t BUCKET_MIN_N = 1ull << 24;  // traces of fewer records keep the full sort
// k_bucket.cu — bucket path of the sort + compaction (keys sorted by key_hi >> HYB_LO only)
size_t bucket_temp_bytes(u32 nchunks);
// sample of the chunk sizes from the extents' granule array: *h_max (host, after a sync) = largest sampled count
u32 bucket_sample_max(const u32* gran, u32 n, u32 gmin_lo, u32 nchunks, void* temp, cudaStream_t st, u32* h_max,
                      u32* samples, u32 want);
u32 bucket_sample_keys_max(const u64* keys, u32 m, u32 shift, u32 nchunks, void* temp, cudaStream_t st, u32* h_max,
                           u32* samples, u32 want);
u32 launch_bucket_compact(u64* keys, u64* stage, u32 m, u32 pos_bits, u32 nchunks, void* temp, u32* total,
                          cudaStream_t st);

// k_util.cu
// per-device launch properties (thread-safe; the shared-memory opt-in is stored per device context)
int dev_sm_count();                                       // SMs of the current device
void smem_optin(const void* kern, size_t bytes);          // cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once
int blocks_per_sm(const void* kern, int threads, size_t smem);  // occupancy (opts in to `smem` first)
size_t scan_u32_temp_bytes(u64 n);
void launch_scan_exclusive_u32(const u32* in, u32* out, u64 n, void* temp, cudaStream_t st);  // out may alias in

// k_sort.cu
void launch_bin_base(const u32* hist, u64* bin_base, u32 npass, cudaStream_t st);
// one LSD pass over keys (and optional u32 values) on digit (key >> shift) & (RADIX-1)
void launch_onesweep(const u64* kin, u64* kout, const u32* vin, u32* vout, u32 m, u32 shift, const u64* bin_base,
                     u64* lookback, u32* tile_ctr, u32 epoch, cudaStream_t st);
u32 sort_tile_keys();
// the same pass without the stable order (the bucket path): counting atomics give the ranks
void launch_partition_pass(const u64* kin, u64* kout, u32 m, u32 shift, const u64* bin_base, u64* lookback,
                           u32* tile_ctr, u32 epoch, cudaStream_t st, bool top = true);
// padded (32-aligned runs) bin bases of one digit histogram; sentinels into kout's pad slots; *mpad (device)
void launch_padded_bin_base(const u32* hist, u64* base, u64* kout, u32* mpad, cudaStream_t st);
inline u32 sort_tiles(u64 m) { return (u32)((m + 2047) / 2048); }  // upper bound (smallest tile: 2048 keys)
// race-list keys: (race key, index) -> histograms for npass digits starting at bit 0
void launch_hist_keys(const u64* keys, u32 m, u32 npass, u32* hist, cudaStream_t st);
void launch_hist_keys_shift(const u64* keys, u32 m, u32 npass, u32 shift, u32* hist, cudaStream_t st);

// k_conflict.cu — see the file header for the three modes.
// Summary of a set of entries at one level (identity = thread within a sub-run, block within a group).
struct Agg {
  u32 mn[3], mx[3];  // per access type: min / max identity (empty: mn = ~0, mx = 0)
  u32 i1, i2;        // identity attaining v1 / v2
  u64 v1, v1b;       // min write value; min write value over identities != i1 (none: ~0)
  u64 v2, v2b;       // max write value; max write value over identities != i2 (none: 0)
};
// Cheap summary: per type min/max identity + min/max write value.  Resolves every flag except "exists a write
// with identity != mine and value != mine" when the set holds >= 2 writer identities and >= 2 distinct values
// (then the query is "unknown" and the check is redone with the exact summary).
struct AggC {
  u32 mn[3], mx[3];
  u64 vlo, vhi;  // min / max write value (empty: ~0 / 0)
};
struct AggQuad {
  Agg a[4];
};
struct AggQuadC {
  AggC a[4];
};
struct ConflictArgs {
  const u64* keys;  // sorted entry keys
  u32 m;            // entries
  const Rec* rec;   // records (gathered by position - rec_pos_base) ...
  const Rec* rec_entry;  // ... or, if set, entry-aligned records (distributed check: fetched from owners)
  u32 rec_pos_base;
  u64 n;
  KeyLayout L;
  u32 ws, ls;
  // outputs (mode 1)
  u32* race_count;
  u64* race_keys;   // canonical sort key per race
  u32* race_vals;   // race index
  struct RaceOut* races;
  u32 race_cap;
  // crossing bookkeeping
  u32* cross_list;   // tiles with a location run crossing a tile boundary
  u32* cross_count;
  u8* tile_flags;    // per tile: bit0 grp head in tile, bit1 grp tail in tile, bit2 sub head, bit3 sub tail,
                     // bit4 cross-in, bit5 cross-out
  void* part;      // per tile AggQuad(C): [0] grp first piece (P), [1] grp last piece (S), [2] sub P, [3] sub S
  void* carry;     // per tile AggQuad(C): [0] grp In, [1] grp Out, [2] sub In, [3] sub Out
  u32* need_exact; // set by cheap-summary tiles that met an unknown benign query
  u32* owner;             // per tile: tile index holding the head of the group that crosses into this tile
  struct Slot* slots;     // per owner tile
  u64 index_base;
  u32 phase;  // modes 2/3: 0 = every crossing piece, 1 = pieces starting a run (crossing out), 2 = the rest
  u32 tdiv;   // > 1: a record's identity is thread / tdiv (precise warp model, inter-warp half)
  const u32* tstart;  // [tiles + 1]: first entry of every tile window (launch_tile_starts)
  u32* work;          // modes 2/3: crossing tiles with work (cross_filter_kernel), count in *work_count
  u32* work_count;
};

struct RaceOut {  // == sesa_race (40 bytes)
  u64 addr, first, second;
  u32 block, interval;
  u8 space, kind, reserved[2];
  u32 epoch;  // kernel launch of the location (multi-launch checks); 0 otherwise
};
static_assert(sizeof(RaceOut) == 40, "race layout");

// per-owner-tile slot for a group crossing tile boundaries
struct Slot {
  u64 x[2];      // min over flagged entries of (position << 32 | entry index) per kind (RW, WW), ~0 = none
  u64 y[2];      // min over partners of x of (position << 32 | entry index) per kind
  u64 head_key;  // key of the group's first entry
  u32 hblock, hinterval;
};

void launch_conflict(int mode, bool exact, const ConflictArgs& a, u32 ntiles_or_list, cudaStream_t st);
void launch_carry(bool exact, const ConflictArgs& a, u32 ntiles, void* temp, cudaStream_t st);
size_t carry_temp_bytes(u32 ntiles);
void launch_cross_emit(const ConflictArgs& a, u32 ntiles, cudaStream_t st);
void launch_permute_races(const RaceOut* in, const u32* order, RaceOut* out, u32 nr, cudaStream_t st);
// out[i] = in[i] with epoch = e (appending one launch's race list to a multi-launch result)
void launch_races_set_epoch(const RaceOut* in, u32 nr, u32 e, RaceOut* out, cudaStream_t st);
void race_rekey_launch(const RaceOut* r, u64 n, const KeyLayout& L, u64* keys, u32* vals, cudaStream_t st);
u32 conflict_tiles(u64 m);
void launch_tile_starts(const ConflictArgs& a, u32 ntiles, u32* tstart, cudaStream_t st);
// benign W/W reporting (k_conflict.cu)
void launch_benign_mark(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, u32* head, u32* wflag,
                        cudaStream_t st);
void launch_benign_gather(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* head,
                          const u32* hscan, const u32* wflag, const u32* wscan, u32* gid, u64* vkey, u32* vidx,
                          cudaStream_t st);
void launch_benign_keys(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* vidx, u32 m3, const u32* gid,
                        int what, u64* keys, cudaStream_t st);
void launch_benign_runs(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* gid, const u32* order,
                        u32 m3, u32* rhead, cudaStream_t st);
void launch_benign_derive(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* order, const u32* rhead,
                          const u32* rscan, u32 m3, Rec* out, u32* dpos, u32* dj, cudaStream_t st);
void launch_benign_min_emit(const ConflictArgs& a, const struct RaceOut* cr, u32 nc, const u32* dpos, const u32* dj,
                            const u32* gid, unsigned long long* slot, cudaStream_t st);

// precise warp model (k_conflict.cu): slots [2 * runs] of (position << 32 | position) minima
void launch_warp_keys(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, u32 ws, u32* head, u32* hkey,
                      cudaStream_t st);
void launch_warp_key2(const u32* head, const u32* hscan, const u32* hkey, u32 m2, u64* key2, u32* val, cudaStream_t st);
void launch_warp_pairs(const u64* comp, const KeyLayout& L, const Rec* rec, const void* ext, u32 ws, const u64* key2,
                       const u32* order, u32 m2, unsigned long long* slot, cudaStream_t st);
void launch_warp_fold(const u64* rkeys, const struct RaceOut* races, u32 nr, const u64* comp, u32 m2,
                      const KeyLayout& L, const u32* hscan, u64 index_base, unsigned long long* slot, cudaStream_t st);
void launch_warp_emit(const ConflictArgs& a, const u32* head, const u32* hscan, const unsigned long long* slot,
                      cudaStream_t st);

// k_compact.cu — keep only entries of locations touched >= 2 times (order preserved); *total = count
size_t compact_temp_bytes(u64 m);
// keys: sorted (m); seg: free buffer of m keys; out: where the result goes (may alias keys, which is dead after);
// returns out
// filter (needs L.wbit): also drop read-only locations (compact_seg_w_kernel); with L.wbit the output is always
// the plain layout (the bit stripped)
u64* launch_compact_multi(const u64* keys, u32 m, const KeyLayout& L, u64* seg, u64* out, void* temp, u32* total,
                          cudaStream_t st, bool filter = false);
// sample whether the write-bit filter pays on these sorted keys (one sync); temp: >= 16 bytes of device memory
bool compact_filter_pays(const u64* keys, u32 m, const KeyLayout& L, void* temp, cudaStream_t st);

// k_expand.cu — cells (block, interval slot, thread); descriptors of slot q are idx[ivoff[q] .. ivoff[q+1])
void launch_flow_count2(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                        u32* cnt, cudaStream_t st);
void launch_flow_write2(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                        const u32* off, Rec* out, cudaStream_t st);

// descriptor-level check (k_expand.cu)
size_t flow_range_bytes(u32 nf);
void launch_flow_ranges(const void* flows, u32 nf, u32 log2G, void* ranges, u32* keep, cudaStream_t st);
void launch_flow_count_sel(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                           const u32* keep, u32* cnt_all, u32* cnt_kept, cudaStream_t st);
void launch_flow_write_sel(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                           const u32* keep, const u32* off_all, const u32* off_kept, Rec* out, u32* orig,
                           cudaStream_t st);
void launch_race_remap(struct RaceOut* races, u32 nr, const u32* orig, cudaStream_t st);

}  // namespace sesa
