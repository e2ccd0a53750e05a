// dist.cu — multi-GPU race check (SURVEY §8a rows a3 "shard + all-to-all" and a7 "gather + merge").
//
// Every race is a property of one location λ (two accesses to the same location), so entries shard by
// owner(λ) = mix64(λ) mod N with no other communication than:
//   X1  all-reduce of the extents summaries (one consistent key layout on every rank) + all-gather of the
//       shard boundaries (global (block, interval) order, global record positions)
//   X2  all-to-all of the 8-byte sort keys (carrying the GLOBAL record position) to their location owners
//   X3  all-to-all of the positions of entries at locations touched >= 2 times (the only ones that can race;
//       2e5 of C5's 1e9) to the ranks holding those records, and X4 the 32-byte records back
//   X5  gather of the (already canonically ordered) per-rank race lists to rank 0, which re-sorts the union.
// The exchange is an interface: NCCL (one process per GPU, grouped ncclSend/ncclRecv over NVLink/NVSwitch) or
// a loopback implementation (W virtual ranks on one GPU, device copies) that runs the same kernels and data
// flow for tests.  Received key blocks are concatenated in source-rank order, so global positions stay
// ascending: the LSD sort's stability then yields the same canonical run order as a 1-GPU check.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <vector>

#include "sesa_internal.h"

using namespace sesa;

namespace sesa {

// ------------------------------------------------------------------------------------------------ partition
// Stable partition of u64 items into W <= 8 buckets.  Warp chunks of 512 items (16 coalesced rows); per-chunk
// bucket counts -> one exclusive scan over the bucket-major count matrix -> writes.  MODE 0: item = sort key,
// bucket = mix64(location run key) mod W.  MODE 1: item = key of a compacted entry, emitted as its global
// position, bucket = owner rank of that position (bases[W+1]); the entry index is written alongside.  MODE 2 =
// MODE 0 with the key formed on the fly from the extents pass's 32-bit granule array (one-granule global records,
// key_hi = g - gmin < 2^32): the key extraction pass (a second 32-byte read per record) is gone, and both
// partition sweeps read 4 instead of 8 bytes per record.
constexpr int PT_ROWS = 16, PT_CHUNK = 32 * PT_ROWS, PT_THREADS = 256;

struct PartArgs {
  const u64* in;
  const u32* gran;  // MODE 2: granule low halves
  u32 gmin_lo;      // MODE 2: low 32 bits of the layout's gminG
  u64 pos_base;     // MODE 2: global position of item 0
  u64 n;
  u32 W;
  int mode;
  KeyLayout L;
  u64 bases[9];
  u32* cnt;        // [W][nchunks]
  const u32* off;  // exclusive scan of cnt
  u64* out;
  u32* out_src;
};

// MODE 2 owner: a 32-bit mix of key_hi scaled to [0, W) (one layout for every rank; MODE 0 is never mixed in)
__device__ __forceinline__ u32 owner32(u32 h, u32 W) {
  h ^= h >> 16, h *= 0x85EBCA6Bu, h ^= h >> 13, h *= 0xC2B2AE35u, h ^= h >> 16;
  return __umulhi(h, W);
}

__device__ __forceinline__ u32 part_bucket(const PartArgs& a, u64 item) {
  // owner = the high half of a 64-bit hash of the location scaled to [0, W) (multiply-shift: a 64-bit modulo by a
  // runtime W is a ~100-instruction emulated division and made both partition sweeps ALU-bound)
  if (a.mode != 1) return (u32)(((sesa_mix(group_of_hi(a.L, item >> a.L.pos_bits)) >> 32) * a.W) >> 32);
  const u64 pos = item & lowmask(a.L.pos_bits);
  u32 r = 0;
  while (r + 1 < a.W && pos >= a.bases[r + 1]) r++;
  return r;
}

template <bool WRITE, int MODE>
__global__ void __launch_bounds__(PT_THREADS) partition_kernel(PartArgs a) {
  // Per row of 32 items a warp multi-split: three ballots of the bucket bits give every lane the mask of its
  // bucket peers (rank = peers before it) and lane d the count of bucket d; lane d keeps bucket d's running
  // offset (a per-bucket ballot loop cost ~100 thread instructions per item).  MODE 0/2 writes: the chunk is
  // staged per bucket in shared memory (chunk-local bases from the count sweep) and leaves in coalesced runs.
  constexpr bool STAGE = WRITE && MODE != 1;
  __shared__ u64 stage[STAGE ? PT_THREADS / 32 : 1][STAGE ? PT_CHUNK : 1];
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  const u64 nch = (a.n + PT_CHUNK - 1) / PT_CHUNK;
  const u64 gw = ((u64)blockIdx.x * PT_THREADS + threadIdx.x) >> 5, nw = ((u64)gridDim.x * PT_THREADS) >> 5;
  u64* st = stage[STAGE ? (threadIdx.x >> 5) : 0];
  const bool own = lane < (int)a.W;  // lane d owns bucket d
  for (u64 c = gw; c < nch; c += nw) {
    // lane d: global offset of bucket d's part of this chunk (write) and its chunk-local staging base
    const u32 mycnt = STAGE && own ? a.cnt[(u64)lane * nch + c] : 0u;
    u32 lbase = mycnt;  // exclusive prefix over the buckets (lanes) of the chunk counts
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) {
      const u32 y = __shfl_up_sync(~0u, lbase, o);
      if (lane >= o) lbase += y;
    }
    lbase -= mycnt;
    const u32 goff = WRITE && own ? a.off[(u64)lane * nch + c] : 0u;
    u32 run = STAGE ? lbase : goff;  // lane d: next slot of bucket d (staging or global)
    const u32 total = __shfl_sync(~0u, lbase + mycnt, 7);
    // every row of the chunk in flight first (the sweep was latency-bound one row at a time)
    u64 items[PT_ROWS];
#pragma unroll
    for (int r = 0; r < PT_ROWS; r++) {
      const u64 i = c * PT_CHUNK + (u64)r * 32 + lane;
      if (MODE == 2) {  // key_hi in the low half until the bucket is known
        items[r] = i >= a.n ? 0ull : (u64)(__ldg(a.gran + i) - a.gmin_lo);
      } else {
        items[r] = i >= a.n ? 0ull : __ldg(a.in + i);
      }
    }
#pragma unroll
    for (int r = 0; r < PT_ROWS; r++) {
      const u64 i = c * PT_CHUNK + (u64)r * 32 + lane;
      const bool valid = i < a.n;
      u64 item = items[r];
      u32 b = 0;
      if (valid) {
        if (MODE == 2) {
          b = owner32((u32)item, a.W);
          item = (item << a.L.pos_bits) | (a.pos_base + i);
        } else {
          b = part_bucket(a, item);
        }
      }
      const unsigned vm = __ballot_sync(~0u, valid), m0 = __ballot_sync(~0u, b & 1u),
                     m1 = __ballot_sync(~0u, b & 2u), m2 = __ballot_sync(~0u, b & 4u);
      const unsigned peers = vm & ((b & 1u) ? m0 : ~m0) & ((b & 2u) ? m1 : ~m1) & ((b & 4u) ? m2 : ~m2);
      const u32 d = (u32)lane;  // the bucket this lane counts
      const unsigned dm = vm & ((d & 1u) ? m0 : ~m0) & ((d & 2u) ? m1 : ~m1) & ((d & 4u) ? m2 : ~m2);
      const u32 slot = __shfl_sync(~0u, run, (int)b) + __popc(peers & lt);
      if (valid && WRITE) {
        if (STAGE) {
          st[slot] = item;
        } else {
          a.out[slot] = MODE != 1 ? item : (item & lowmask(a.L.pos_bits));
          if (a.out_src) a.out_src[slot] = (u32)i;
        }
      }
      if (own) run += __popc(dm);
    }
    if (STAGE) {
      u32 LB[8], GO[8];
#pragma unroll
      for (int q = 0; q < 8; q++) LB[q] = __shfl_sync(~0u, lbase, q), GO[q] = __shfl_sync(~0u, goff, q);
      __syncwarp();
      for (u32 j = lane; j < total; j += 32) {  // bucket of slot j: the last one whose base is <= j
        u32 dst = 0;
#pragma unroll
        for (int q = 0; q < 8; q++)
          if (q < (int)a.W && j >= LB[q]) dst = GO[q] + (j - LB[q]);
        a.out[dst] = st[j];
      }
      __syncwarp();
    }
    if (!WRITE && own) a.cnt[(u64)lane * nch + c] = run;
  }
}

__global__ void bucket_totals_kernel(const u32* cnt, const u32* off, u64 nch, u32 W, u64* tot) {
  const u32 d = threadIdx.x;
  // bucket d occupies [off[d*nch], off[d*nch + nch-1] + cnt[d*nch + nch-1]) of the bucket-major output
  if (d < W) tot[d] = nch ? (u64)off[(u64)d * nch + nch - 1] + cnt[(u64)d * nch + nch - 1] - off[(u64)d * nch] : 0ull;
}

__global__ void gather_records_kernel(const Rec* __restrict__ rec, const u64* __restrict__ pos, u64 base, u64 n,
                                      Rec* __restrict__ out) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = rec[pos[i] - base];
}

__global__ void scatter_records_kernel(const Rec* __restrict__ in, const u32* __restrict__ dst, u64 n,
                                       Rec* __restrict__ out) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[dst[i]] = in[i];
}

}  // namespace sesa

// ------------------------------------------------------------------------------------------------ state
struct RankBufs {
  DevBuf pcnt, poff, ptmp, send, recv, src, req, reqin, recsend, recback, rec_entry, tot, rkeys, rvals, races, ag, gran;
};

struct DistState {
  ncclComm_t comm = nullptr;
  RankBufs b;
};

// per-rank host-side values exchanged in X1
struct RankInfo {
  unsigned long long n, base, first_b, first_i, last_b, last_i, bad;  // bad: global index or ~0
  unsigned long long fail;                                            // status of the rank's P1 (0 = ok)
};

static bool partition(sesa_trace* t, RankBufs& B, const u64* in, u64 n, u32 W, int mode, const u64* bases,
                      u64* out_tot /*[W]*/, const u32* gran = nullptr, u64 pos_base = 0) {
  PartArgs a;
  memset(&a, 0, sizeof a);
  a.in = in;
  a.gran = gran;
  a.gmin_lo = (u32)t->layout.gminG;
  a.pos_base = pos_base;
  a.n = n;
  a.W = W;
  a.mode = mode;
  a.L = t->layout;
  for (u32 i = 0; i <= W && bases; i++) a.bases[i] = bases[i];
  const u64 nch = (n + PT_CHUNK - 1) / PT_CHUNK;
  const u64 ncnt = std::max<u64>(nch * W, 1);
  if (!t->grow(B.pcnt, ncnt * 4, "part counts") || !t->grow(B.poff, ncnt * 4, "part offsets") ||
      !t->grow(B.ptmp, scan_u32_temp_bytes(ncnt), "part scan") || !t->grow(B.send, std::max<u64>(n, 1) * 8, "send") ||
      !t->grow(B.src, std::max<u64>(n, 1) * 4, "src") || !t->grow(B.tot, 8 * 8, "totals"))
    return false;
  a.cnt = (u32*)B.pcnt.p;
  a.off = (u32*)B.poff.p;
  a.out = (u64*)B.send.p;
  a.out_src = mode == 1 ? (u32*)B.src.p : nullptr;
  if (n) {
    const unsigned grid = (unsigned)std::min<u64>((nch + 7) / 8, (u64)t->num_sms * 8);
    t->launch_begin("owner_partition");  // (3 kernels + the scan's one: kernels_of counts them)
    auto sweep = [&](bool write) {
      if (mode == 2) write ? partition_kernel<true, 2><<<grid, PT_THREADS, 0, t->stream>>>(a)
                           : partition_kernel<false, 2><<<grid, PT_THREADS, 0, t->stream>>>(a);
      else if (mode == 1) write ? partition_kernel<true, 1><<<grid, PT_THREADS, 0, t->stream>>>(a)
                                : partition_kernel<false, 1><<<grid, PT_THREADS, 0, t->stream>>>(a);
      else write ? partition_kernel<true, 0><<<grid, PT_THREADS, 0, t->stream>>>(a)
                 : partition_kernel<false, 0><<<grid, PT_THREADS, 0, t->stream>>>(a);
    };
    sweep(false);
    launch_scan_exclusive_u32((u32*)B.pcnt.p, (u32*)B.poff.p, nch * W, B.ptmp.p, t->stream);
    sweep(true);
    bucket_totals_kernel<<<1, 32, 0, t->stream>>>((u32*)B.pcnt.p, (u32*)B.poff.p, nch, W, (u64*)B.tot.p);
    t->launch_end(24.0 * (double)n);
    if (!t->cuda_ok(cudaMemcpyAsync(out_tot, B.tot.p, W * 8, cudaMemcpyDeviceToHost, t->stream), "totals")) return false;
  } else {
    for (u32 i = 0; i < W; i++) out_tot[i] = 0;
  }
  return t->sync_check("partition");
}

// ------------------------------------------------------------------------------------------------ exchange
// One exchange = every rank sends count[r][p] elements (elem bytes) of its send buffer (bucket-major) to rank p,
// and receives, concatenated in source-rank order, into its recv buffer.
struct Exchanger {
  virtual ~Exchanger() {}
  virtual int world() const = 0;
  // host-side all-gather of a per-rank POD value
  virtual bool allgather(sesa_trace* t, const void* mine, void* all, size_t bytes) = 0;
  // send[p] counts (elements) -> recv from each peer; offsets computed by the caller
  virtual bool alltoall(sesa_trace* t, const void* send, const u64* scnt, void* recv, const u64* rcnt, size_t elem) = 0;
};

struct NcclExchanger : Exchanger {
  ncclComm_t comm;
  int rank_, world_;
  DevBuf& tmp;  // staging of the host all-gathers (owned by the handle's DistState, freed by destroy)
  NcclExchanger(ncclComm_t c, int r, int w, DevBuf& t) : comm(c), rank_(r), world_(w), tmp(t) {}
  int world() const override { return world_; }
  bool nccl_ok(sesa_trace* t, ncclResult_t r, const char* what) {
    if (r == ncclSuccess) return true;
    t->fail(SESA_ENCCL, "%s: %s", what, ncclGetErrorString(r));
    return false;
  }
  bool allgather(sesa_trace* t, const void* mine, void* all, size_t bytes) override {
    if (!t->grow(tmp, bytes * (world_ + 1), "allgather")) return false;
    char* d = (char*)tmp.p;
    cudaMemcpyAsync(d + bytes * world_, mine, bytes, cudaMemcpyHostToDevice, t->stream);
    if (!nccl_ok(t, ncclAllGather(d + bytes * world_, d, bytes, ncclUint8, comm, t->stream), "ncclAllGather")) return false;
    cudaMemcpyAsync(all, d, bytes * world_, cudaMemcpyDeviceToHost, t->stream);
    return t->sync_check("allgather");
  }
  bool alltoall(sesa_trace* t, const void* send, const u64* scnt, void* recv, const u64* rcnt, size_t elem) override {
    u64 so = 0, ro = 0;
    if (!nccl_ok(t, ncclGroupStart(), "ncclGroupStart")) return false;
    for (int p = 0; p < world_; p++) {
      if (scnt[p] && !nccl_ok(t, ncclSend((const char*)send + so * elem, scnt[p] * elem, ncclUint8, p, comm, t->stream),
                              "ncclSend"))
        return false;
      if (rcnt[p] && !nccl_ok(t, ncclRecv((char*)recv + ro * elem, rcnt[p] * elem, ncclUint8, p, comm, t->stream),
                              "ncclRecv"))
        return false;
      so += scnt[p];
      ro += rcnt[p];
    }
    if (!nccl_ok(t, ncclGroupEnd(), "ncclGroupEnd")) return false;
    return t->sync_check("alltoall");
  }
};

// ------------------------------------------------------------------------------------------------ the check
// Runs the collective check for `R` ranks whose handles are ts[0..R) (one real rank with NCCL: R = 1 and
// my_rank = its rank; loopback: R = world virtual ranks on this GPU).  Phases are executed for every local rank
// before each exchange; for loopback the exchange is performed by device copies between the local handles.
struct LoopbackCtx {
  std::vector<sesa_trace*> ts;
};

static bool fail_all(std::vector<sesa_trace*>& ts, const sesa_trace* src) {
  for (auto* t : ts)
    if (t != src) t->status = src->status, t->err = src->err;
  return false;
}

struct RankIO {
  const Rec* rec;
  u64 n, index_base;
};

// A local failure must not leave the peers blocked in the next collective (one process per GPU): every exchange
// first all-gathers, with the count rows, one status word per rank, and all ranks fail together if any failed.
// `local_ok` = this rank's phase before the exchange succeeded (its send buffers are valid).
static bool agree(sesa_trace* t, int p, u64 st, u64 local_ok) {
  if (st == SESA_OK) return true;
  if (local_ok) t->fail((sesa_status)st, "rank %d failed before the exchange (status %s)", p, sesa_status_str((sesa_status)st));
  return false;
}

// exchange helper covering both modes: per local rank r, send buffers/counts -> recv buffers/counts
static bool exchange(std::vector<sesa_trace*>& ts, Exchanger* ex, const std::vector<const void*>& send,
                     const std::vector<std::vector<u64>>& scnt, std::vector<DevBuf*>& recv, std::vector<std::vector<u64>>& rcnt,
                     size_t elem, const char* what, bool local_ok = true) {
  const int W = ex ? ex->world() : (int)ts.size();
  const int R = (int)ts.size();
  rcnt.assign(R, std::vector<u64>(W, 0));
  if (!ex && !local_ok) return false;  // loopback: every virtual rank already carries the failure (fail_all)
  if (ex) {  // real ranks: one local handle; counts + status by all-gather of the count rows
    sesa_trace* t = ts[0];
    std::vector<u64> row(W + 1, 0), all((size_t)W * (W + 1));
    if (local_ok) std::copy(scnt[0].begin(), scnt[0].end(), row.begin());
    row[W] = local_ok ? (u64)SESA_OK : (u64)(t->status != SESA_OK ? t->status : SESA_ECUDA);
    if (!ex->allgather(t, row.data(), all.data(), (W + 1) * 8)) return false;
    bool ok = true;
    for (int p = 0; p < W; p++) ok = agree(t, p, all[(size_t)p * (W + 1) + W], local_ok && ok) && ok;
    if (!ok || !local_ok) return false;
    int me = t->rank;
    u64 tot = 0;
    for (int p = 0; p < W; p++) rcnt[0][p] = all[(size_t)p * (W + 1) + me], tot += rcnt[0][p];
    if (!t->grow(*recv[0], std::max<u64>(tot, 1) * elem + 64, what)) return false;
    u64 sent = 0;  // bytes that cross NVLink (to other ranks)
    for (int p = 0; p < W; p++)
      if (p != me) sent += scnt[0][p] * elem;
    t->launch_begin("alltoall");
    const bool ok2 = ex->alltoall(t, send[0], scnt[0].data(), recv[0]->p, rcnt[0].data(), elem);
    t->launch_end((double)sent);
    return ok2;
  }
  // loopback: rank r receives from every s, in source order
  if (getenv("SESA_SYNC_DEBUG"))
    for (int r = 0; r < R; r++)
      for (int p = 0; p < W; p++) fprintf(stderr, "[sesa debug] %s scnt[%d][%d] = %llu\n", what, r, p, (unsigned long long)scnt[r][p]);
  for (int r = 0; r < R; r++) {
    u64 tot = 0;
    for (int s = 0; s < R; s++) rcnt[r][s] = scnt[s][r], tot += scnt[s][r];
    if (!ts[r]->grow(*recv[r], std::max<u64>(tot, 1) * elem + 64, what)) return fail_all(ts, ts[r]);
  }
  for (int r = 0; r < R; r++) {
    u64 ro = 0;
    for (int s = 0; s < R; s++) {
      u64 so = 0;
      for (int q = 0; q < r; q++) so += scnt[s][q];
      if (scnt[s][r])
        cudaMemcpyAsync((char*)recv[r]->p + ro * elem, (const char*)send[s] + so * elem, scnt[s][r] * elem,
                        cudaMemcpyDeviceToDevice, ts[0]->stream);
      ro += scnt[s][r];
    }
  }
  return ts[0]->sync_check(what) || fail_all(ts, ts[0]);
}

static sesa_status dist_check(std::vector<sesa_trace*>& ts, std::vector<RankIO>& io, Exchanger* ex) {
  const int R = (int)ts.size();
  const int W = ex ? ex->world() : R;
  for (int r = 0; r < R; r++) ts[r]->begin_check(io[r].n);
  // --- P1: extents per rank (a local failure is carried into X1, so that no peer waits for this rank)
  std::vector<bool> p1ok(R, true);
  for (int r = 0; r < R; r++) {
    if (io[r].n && !ts[r]->check_records_ptr((const sesa_access*)io[r].rec, io[r].n)) p1ok[r] = false;
    // (+ the 32-bit granule array: the owner partition forms the keys from it when the global layout allows)
    else if (!ts[r]->grow(ts[r]->ds->b.gran, std::max<u64>(io[r].n, 1) * 4, "granules") ||
             !ts[r]->step_extents(io[r].rec, io[r].n, false, (u32*)ts[r]->ds->b.gran.p))
      p1ok[r] = false;
    if (!p1ok[r] && !ex) return fail_all(ts, ts[r]), ts[r]->status;
  }
  // --- X1: summaries + shard boundaries
  std::vector<RankInfo> infos(W);
  std::vector<Summary> sums(W);
  for (int r = 0; r < R; r++) {
    RankInfo ri;
    memset(&ri, 0, sizeof ri);
    ri.n = io[r].n;
    ri.base = io[r].index_base;
    ri.fail = p1ok[r] ? 0ull : (unsigned long long)(ts[r]->status != SESA_OK ? ts[r]->status : SESA_ECUDA);
    ri.bad = !p1ok[r] || ts[r]->h_summary.bad_index == ~0ull ? ~0ull : io[r].index_base + ts[r]->h_summary.bad_index;
    if (io[r].n && p1ok[r]) {
      sesa_access f, l;
      cudaMemcpy(&f, io[r].rec, 32, cudaMemcpyDeviceToHost);
      cudaMemcpy(&l, io[r].rec + io[r].n - 1, 32, cudaMemcpyDeviceToHost);
      ri.first_b = f.block, ri.first_i = f.interval, ri.last_b = l.block, ri.last_i = l.interval;
    }
    if (ex) {
      if (!ex->allgather(ts[0], &ri, infos.data(), sizeof ri)) return ts[0]->status;
      bool ok = true;
      for (int p = 0; p < W; p++) ok = agree(ts[0], p, infos[p].fail, p1ok[0] && ok) && ok;
      if (!ok || !p1ok[0]) return ts[0]->status;
      if (!ex->allgather(ts[0], &ts[0]->h_summary, sums.data(), sizeof(Summary))) return ts[0]->status;
    } else {
      infos[r] = ri;
      sums[r] = ts[r]->h_summary;
    }
  }
  Summary S = sums[0];
  u64 bad = ~0ull;
  for (int p = 0; p < W; p++) bad = std::min<u64>(bad, infos[p].bad);
  if (bad != ~0ull) {
    for (int r = 0; r < R; r++) {
      const u64 b0 = io[r].index_base;
      if (bad >= b0 && bad < b0 + io[r].n) ts[r]->report_bad((const sesa_access*)io[r].rec, bad - b0, bad);
      else ts[r]->fail(SESA_EINVAL, "record %llu invalid (on another rank)", (unsigned long long)bad);
    }
    return SESA_EINVAL;
  }
  // OOB report (NEXT-1): every rank contributes (count, global first index, that record); all ranks merge
  {
    struct OobPart {
      u64 count, first;
      sesa_access rec;
    };
    std::vector<OobPart> parts(W);
    for (int r = 0; r < R; r++) {
      OobPart op;
      memset(&op, 0, sizeof op);
      const Summary& h = ts[r]->h_summary;
      op.count = h.oob_count;
      op.first = h.oob_count ? io[r].index_base + h.oob_first : ~0ull;
      if (h.oob_count) cudaMemcpy(&op.rec, io[r].rec + h.oob_first, 32, cudaMemcpyDeviceToHost);
      if (ex) {
        if (!ex->allgather(ts[0], &op, parts.data(), sizeof op)) return ts[0]->status;
      } else {
        parts[r] = op;
      }
    }
    sesa_oob_report rep;
    memset(&rep, 0, sizeof rep);
    rep.first_index = ~0ull;
    for (int p = 0; p < W; p++) {
      rep.n_oob += parts[p].count;
      if (parts[p].count && parts[p].first < rep.first_index) rep.first_index = parts[p].first, rep.first = parts[p].rec;
    }
    for (int r = 0; r < R; r++) ts[r]->oob = rep, ts[r]->have_oob = true;
  }
  for (int p = 1; p < W; p++) {
    const Summary& q = sums[p];
    S.entries += q.entries, S.multi += q.multi, S.unsorted |= q.unsorted;
    for (int sp = 0; sp < 2; sp++) {
      if (!q.count[sp]) continue;
      if (!S.count[sp]) {
        S.gmin[sp] = q.gmin[sp], S.gmax[sp] = q.gmax[sp], S.bmin[sp] = q.bmin[sp], S.bmax[sp] = q.bmax[sp];
        S.imin[sp] = q.imin[sp], S.imax[sp] = q.imax[sp];
      } else {
        S.gmin[sp] = std::min(S.gmin[sp], q.gmin[sp]), S.gmax[sp] = std::max(S.gmax[sp], q.gmax[sp]);
        S.bmin[sp] = std::min(S.bmin[sp], q.bmin[sp]), S.bmax[sp] = std::max(S.bmax[sp], q.bmax[sp]);
        S.imin[sp] = std::min(S.imin[sp], q.imin[sp]), S.imax[sp] = std::max(S.imax[sp], q.imax[sp]);
      }
      S.count[sp] += q.count[sp];
    }
  }
  // global (block, interval) order across shard boundaries; shards must be contiguous in index order
  u64 ntot = 0, base0 = infos[0].base;
  int prev = -1;
  for (int p = 0; p < W; p++) {
    if (infos[p].base != base0 + ntot) {
      for (auto* t : ts) t->fail(SESA_EINVAL, "index_base of rank %d is %llu, expected %llu (exclusive prefix)", p,
                                 (unsigned long long)infos[p].base, (unsigned long long)(base0 + ntot));
      return SESA_EINVAL;
    }
    ntot += infos[p].n;
    if (!infos[p].n) continue;
    if (prev >= 0 && (infos[p].first_b < infos[prev].last_b ||
                      (infos[p].first_b == infos[prev].last_b && infos[p].first_i < infos[prev].last_i)))
      S.unsorted = 1;
    prev = p;
  }
  if (S.entries >= (1ull << 31) || ntot >= (1ull << 31)) {
    for (auto* t : ts) t->fail(SESA_ERANGE, "%llu entries / %llu records >= 2^31 (ABI v1 limit)",
                               (unsigned long long)S.entries, (unsigned long long)ntot);
    return SESA_ERANGE;
  }
  std::vector<u64> bases(W + 1);
  for (int p = 0; p < W; p++) bases[p] = infos[p].base - base0;
  bases[W] = ntot;
  for (int r = 0; r < R; r++) {
    if (!ts[r]->make_layout(S, std::max<u64>(ntot, 1))) return fail_all(ts, ts[r]), SESA_ERANGE;
    ts[r]->info.n_entries = S.entries;
    ts[r]->info.sort_bits = ts[r]->layout.sort_bits;
    ts[r]->info.pos_bits = ts[r]->layout.pos_bits;
  }
  // --- P2: keys with global positions, partitioned by location owner
  std::vector<std::vector<u64>> scnt(R, std::vector<u64>(W)), rcnt;
  std::vector<const void*> sendp(R);
  std::vector<DevBuf*> recvb(R);
  bool ok = true;  // this process's ranks completed the phase (NCCL: carried into the next exchange)
  for (int r = 0; r < R && ok; r++) {
    sesa_trace* t = ts[r];
    const u64 mloc = t->h_summary.entries;
    sendp[r] = t->ds->b.send.p;
    recvb[r] = &t->b_keys[1];  // received keys land in b_keys[1], then are copied/swapped into b_keys[0]
    const KeyLayout& L = t->layout;
    const bool fused = S.multi == 0 && !L.both && L.single_space == SP_GLOBAL && L.lowG == 0 && L.sort_bits <= 32;
    if (fused)  // keys formed from the granule array inside the partition sweeps
      ok = partition(t, t->ds->b, nullptr, mloc, W, 2, nullptr, scnt[r].data(), (const u32*)t->ds->b.gran.p,
                     io[r].index_base - base0);
    else
      ok = t->step_extract(io[r].rec, io[r].n, mloc, io[r].index_base - base0, S.multi != 0) &&
           partition(t, t->ds->b, (const u64*)t->b_keys[0].p, mloc, W, 0, nullptr, scnt[r].data());
    sendp[r] = t->ds->b.send.p;
    if (!ok) fail_all(ts, t);
  }
  // --- X2: keys to their owners
  if (!exchange(ts, ex, sendp, scnt, recvb, rcnt, 8, "key exchange", ok)) return ts[0]->status;
  // --- P3: local sort + compaction of the received keys; requests for the records of multi-entry locations
  std::vector<u64*> comp(R);
  std::vector<u32> m2(R);
  std::vector<std::vector<u64>> qcnt(R, std::vector<u64>(W)), qrcnt;
  std::vector<DevBuf*> reqb(R);
  for (int r = 0; r < R && ok; r++) {
    sesa_trace* t = ts[r];
    u64 mr = 0;
    for (int s = 0; s < W; s++) mr += rcnt[r][s];
    std::swap(t->b_keys[0], t->b_keys[1]);  // received keys -> b_keys[0]
    int cur = 0;
    bool used = false;  // the bucket path on the received keys when their granules spread evenly (C5)
    ok = t->grow(t->b_keys[1], mr * 8 + 64, "keys") && t->try_bucket_keys(mr, &comp[r], &m2[r], &used) &&
         (used || (t->step_hist(mr) && t->step_sort(mr, &cur) && t->step_compact(cur, mr, &comp[r], &m2[r]))) &&
         partition(t, t->ds->b, comp[r], m2[r], W, 1, bases.data(), qcnt[r].data());
    sendp[r] = t->ds->b.send.p;
    reqb[r] = &t->ds->b.reqin;
    if (!ok) fail_all(ts, t);
  }
  // --- X3: positions to the record owners
  if (!exchange(ts, ex, sendp, qcnt, reqb, qrcnt, 8, "request exchange", ok)) return ts[0]->status;
  // --- P4: owners gather the requested records
  std::vector<std::vector<u64>> bcnt, brcnt;
  bcnt.assign(R, std::vector<u64>(W));
  std::vector<DevBuf*> backb(R);
  for (int r = 0; r < R; r++) {
    sesa_trace* t = ts[r];
    u64 nq = 0;
    for (int s = 0; s < W; s++) nq += qrcnt[r][s], bcnt[r][s] = qrcnt[r][s];
    if (!t->grow(t->ds->b.recsend, std::max<u64>(nq, 1) * 32, "record send")) {
      ok = false;
      fail_all(ts, t);
      break;
    }
    if (nq) {
      t->launches++;
      gather_records_kernel<<<(unsigned)((nq + 255) / 256), 256, 0, t->stream>>>(
          io[r].rec, (const u64*)t->ds->b.reqin.p, io[r].index_base - base0, nq, (Rec*)t->ds->b.recsend.p);
    }
    sendp[r] = t->ds->b.recsend.p;
    backb[r] = &t->ds->b.recback;
  }
  // --- X4: records back to the requesters (in the order of their request buffers)
  if (!exchange(ts, ex, sendp, bcnt, backb, brcnt, 32, "record exchange", ok)) return ts[0]->status;
  // --- P5: entry-aligned records, conflict tiles, local canonical race order
  std::vector<std::vector<u64>> racn(R, std::vector<u64>(W, 0)), racrn;
  for (int r = 0; r < R && ok; r++) {
    sesa_trace* t = ts[r];
    RankBufs& B = t->ds->b;
    sendp[r] = t->b_races_sorted.p;
    recvb[r] = &B.races;
    if (!t->grow(B.rec_entry, std::max<u32>(m2[r], 1) * 32, "entry records")) {
      ok = false;
      fail_all(ts, t);
      break;
    }
    if (m2[r]) {
      t->launches++;
      scatter_records_kernel<<<(m2[r] + 255) / 256, 256, 0, t->stream>>>((const Rec*)B.recback.p, (const u32*)B.src.p,
                                                                          m2[r], (Rec*)B.rec_entry.p);
    }
    ok = t->step_conflict(comp[r], m2[r], nullptr, 0, (const Rec*)B.rec_entry.p, base0) &&
         t->step_benign(comp[r], m2[r], nullptr, base0, (const Rec*)B.rec_entry.p) &&
         t->grow(t->b_races_sorted, (size_t)std::max((u32)t->n_races, 1u) * sizeof(RaceOut), "sorted races") &&
         t->step_race_sort((u32)t->n_races, (RaceOut*)t->b_races.p, (u64*)t->b_rkeys[0].p, (u32*)t->b_rvals[0].p,
                           (u64*)t->b_rkeys[1].p, (u32*)t->b_rvals[1].p, (RaceOut*)t->b_races_sorted.p) &&
         t->sync_check("local races");
    racn[r][0] = t->n_races;  // everything goes to rank 0
    sendp[r] = t->b_races_sorted.p;
    if (!ok) fail_all(ts, t);
  }
  // --- X5: race lists to rank 0 (rank 0 receives every rank's list, in rank order), then one canonical sort
  if (!exchange(ts, ex, sendp, racn, recvb, racrn, sizeof(RaceOut), "race gather", ok)) return ts[0]->status;
  for (int r = 0; r < R; r++) {
    sesa_trace* t = ts[r];
    const bool is0 = (ex ? t->rank : r) == 0;
    t->n_races = 0;
    if (is0) {
      u64 nr = 0;
      for (int s = 0; s < W; s++) nr += racrn[r][s];
      RankBufs& B = t->ds->b;
      if (!t->grow(B.rkeys, std::max<u64>(nr, 1) * 16, "race keys") || !t->grow(B.rvals, std::max<u64>(nr, 1) * 8, "race vals") ||
          !t->grow(t->b_dist_races, std::max<u64>(nr, 1) * sizeof(RaceOut), "races"))
        return fail_all(ts, t), t->status;
      if (nr) {
        t->launches++;
        race_rekey_launch((const RaceOut*)B.races.p, nr, t->layout, (u64*)B.rkeys.p, (u32*)B.rvals.p, t->stream);
        if (!t->step_race_sort((u32)nr, (const RaceOut*)B.races.p, (u64*)B.rkeys.p, (u32*)B.rvals.p,
                               (u64*)B.rkeys.p + nr, (u32*)B.rvals.p + nr, (RaceOut*)t->b_dist_races.p))
          return fail_all(ts, t), t->status;
      }
      t->n_races = nr;
    }
    if (!t->sync_check("race merge")) return fail_all(ts, t), t->status;
    t->info.n_races = t->n_races;
    t->info.launches = t->launches;
    t->collect_prof();
    t->info.n_stats = (u32)t->stats.size();
    t->have_result = true;
  }
  return SESA_OK;
}

// ------------------------------------------------------------------------------------------------ handle glue
sesa_status sesa_trace::check_dist(const sesa_access* d_rec, uint64_t n, uint64_t index_base) {
  if (world == 1) {  // one rank owns every location: nothing to exchange, the single-GPU pipeline is the check
    const sesa_status s = check_device(d_rec, n, index_base);
    if (s == SESA_OK) std::swap(b_dist_races, b_races_sorted);  // rank 0's merged list lives in b_dist_races
    return s;
  }
  std::vector<sesa_trace*> ts = {this};
  std::vector<RankIO> io = {{(const Rec*)d_rec, n, index_base}};
  NcclExchanger ex(ds->comm, rank, world, ds->b.ag);
  const sesa_status s = dist_check(ts, io, &ex);
  if (s != SESA_OK && status == SESA_OK) status = s;
  return status;
}

void sesa_trace::destroy_dist() {
  if (!ds) return;
  RankBufs& B = ds->b;
  for (DevBuf* b : {&B.pcnt, &B.poff, &B.ptmp, &B.send, &B.recv, &B.src, &B.req, &B.reqin, &B.recsend, &B.recback,
                    &B.rec_entry, &B.tot, &B.rkeys, &B.rvals, &B.races, &B.ag, &B.gran})
    if (b->p) cudaFree(b->p), b->p = nullptr;
  if (ds->comm) ncclCommDestroy(ds->comm);
  delete ds;
  ds = nullptr;
}

extern "C" {

sesa_status sesa_nccl_unique_id(uint8_t* out_id) {
  if (!out_id) return SESA_EINVAL;
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return SESA_ENCCL;
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId");
  memcpy(out_id, &id, 128);
  return SESA_OK;
}

sesa_status sesa_trace_create_dist(const sesa_config* cfg, int rank, int world, const uint8_t* uid, sesa_trace** out) {
  if (!out) return SESA_EINVAL;
  *out = nullptr;
  if (!uid || world < 1 || world > 8 || rank < 0 || rank >= world) return SESA_EINVAL;
  sesa_trace* t = nullptr;
  sesa_status s = sesa_trace_create(cfg, &t);
  if (s != SESA_OK) return s;
  t->dist = true;
  t->rank = rank;
  t->world = world;
  t->ds = new DistState();
  ncclUniqueId id;
  memcpy(&id, uid, 128);
  if (ncclCommInitRank(&t->ds->comm, world, id, rank) != ncclSuccess) {
    t->ds->comm = nullptr;
    sesa_trace_destroy(t);
    return SESA_ENCCL;
  }
  *out = t;
  return SESA_OK;
}

// Test/diagnostic entry: the distributed check with `world` virtual ranks on the current GPU (loopback exchange).
// Rank r owns records [offs[r], offs[r+1]) of d_records.  The merged race list is retrieved with
// sesa_races_get(t, ...) on the returned primary handle t (created here; destroy with sesa_trace_destroy).
sesa_status sesa_race_check_loopback(const sesa_config* cfg, const sesa_access* d_records, const uint64_t* offs,
                                     int world, uint64_t index_base, void* stream, sesa_trace** out) {
  if (!out || !offs || world < 1 || world > 8) return SESA_EINVAL;
  *out = nullptr;
  std::vector<sesa_trace*> ts(world, nullptr);
  for (int r = 0; r < world; r++) {
    sesa_status s = sesa_trace_create(cfg, &ts[r]);
    if (s != SESA_OK) {
      for (auto* t : ts) sesa_trace_destroy(t);
      return s;
    }
    ts[r]->stream = (cudaStream_t)stream;
    ts[r]->ds = new DistState();
  }
  std::vector<RankIO> io(world);
  for (int r = 0; r < world; r++)
    io[r] = {(const Rec*)(d_records + offs[r]), offs[r + 1] - offs[r], index_base + offs[r]};
  const sesa_status s = dist_check(ts, io, nullptr);
  // rank 0's handle carries the merged list; expose it as a regular single-GPU result
  sesa_trace* t0 = ts[0];
  if (s == SESA_OK) std::swap(t0->b_races_sorted, t0->b_dist_races);
  for (int r = 1; r < world; r++) sesa_trace_destroy(ts[r]);
  *out = t0;
  return s == SESA_OK ? SESA_OK : t0->status;
}

}  // extern "C"
