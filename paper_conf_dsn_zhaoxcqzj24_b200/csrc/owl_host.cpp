/*
 * owl_host.cpp — the C ABI of libowl (include/owl.h): context and segment registry (A1), Myers slot
 * assignment and evidence bookkeeping (A4), build orchestration with capacity regrowth,
 * canonical export, diff (A5), the kernel-leak test and leak localization (A7) around
 * the KS kernels (A6), and the multi-GPU partition / absorb entry points.  Every step that touches records
 * or cells runs in the CUDA kernels of owl_fold.cu / owl_tables.cu / owl_ks.cu / owl_exchange.cu; this
 * file only marshals, schedules and sorts small host arrays.
 */
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <chrono>
#include <map>
#include <memory>
#include <string>
#include <tuple>
#include <vector>

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "owl.h"
#include "owl_internal.h"
#include "owl_myers.h"

#define OWL_API extern "C" __attribute__((visibility("default")))

/* NVTX range around an ABI call (visible in nsys / ncu timelines; free when no tool is attached) */
struct OwlRange {
  explicit OwlRange(const char* name) { nvtxRangePushA(name); }
  ~OwlRange() { nvtxRangePop(); }
};
#define OWL_RANGE() OwlRange owl_range_(__func__)

namespace {

thread_local std::string g_err;

owl_status fail(owl_status s, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

owl_status cuda_fail(cudaError_t e, const char* what) {
  if (e == cudaErrorMemoryAllocation) return fail(OWL_ERR_OUT_OF_MEMORY, "%s: out of device memory", what);
  return fail(OWL_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CUDA_TRY(expr, what)                  \
  do {                                        \
    cudaError_t _e = (expr);                  \
    if (_e != cudaSuccess) return cuda_fail(_e, what); \
  } while (0)

uint64_t next_pow2(uint64_t v) {
  uint64_t p = 1;
  while (p < v) p <<= 1;
  return p;
}

struct RemoteRun {
  uint32_t cls;
  std::vector<uint64_t> kids;
};

}  // namespace

struct owl_ctx {
  int device = 0;
  int n_sm = 148;
  cudaStream_t stream = nullptr;
  owl_config cfg{};
  std::map<std::pair<uint32_t, uint32_t>, owl_segment> segs; /* (run, seq) -> segment */
  std::map<uint32_t, RemoteRun> remote;
  FoldStatus* d_status = nullptr;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  cudaStream_t copy_stream = nullptr; /* host-record staging (fold_pass) */
  uint64_t cap_hint[T_NUM] = {0, 0, 0, 0};
  /* stats */
  uint64_t fold_launches = 0;
  double last_fold_ms = 0;
  uint64_t last_fold_records = 0;
  double total_fold_ms = 0;
  uint64_t total_fold_records = 0;
};

/* The evidence's slot list: ordered slot ids, kernel id and invocation count per slot id. */
struct SlotState {
  std::vector<uint32_t> order;
  std::vector<uint64_t> kid, count;
  uint32_t n_runs = 0;
};

struct owl_adcfg {
  owl_ctx* ctx = nullptr;
  uint32_t cls = 0;
  int64_t max_run = -1;
  SlotState slots;
  DevTable tab[T_NUM] = {};
  SortedTable sorted[T_NUM];
  bool sorted_ok = false;
  uint64_t n_records = 0;
  ExchangeCell* send = nullptr;
  ~owl_adcfg() {
    for (int t = 0; t < T_NUM; ++t) {
      owl_table_free(&tab[t]);
      owl_sorted_free(&sorted[t]);
    }
    if (send) owl_dev_free(send);
  }
};

namespace {

/* A4: merge one run's kernel sequence into the slot list with Myers; returns the slot of
   each of the run's invocations (in seq order). */
std::vector<uint32_t> slot_merge(SlotState& s, const std::vector<uint32_t>& seqs, const std::vector<uint64_t>& kids) {
  std::vector<uint32_t> out(seqs.size());
  if (s.n_runs == 0) { /* the first run: slots are its invocation indices */
    uint32_t mx = 0;
    for (uint32_t q : seqs) mx = std::max(mx, q + 1);
    s.kid.assign(mx, 0);
    s.count.assign(mx, 0);
    for (size_t i = 0; i < seqs.size(); ++i) {
      s.kid[seqs[i]] = kids[i];
      s.count[seqs[i]] = 1;
      s.order.push_back(seqs[i]);
      out[i] = seqs[i];
    }
    s.n_runs = 1;
    return out;
  }
  std::vector<uint64_t> a;
  for (uint32_t sl : s.order) a.push_back(s.kid[sl]);
  std::vector<OwlEdit> ops = owl_myers(a, kids);
  std::vector<uint32_t> order;
  for (const OwlEdit& o : ops) {
    if (o.op == OWL_EDIT_MATCH) {
      const uint32_t sl = s.order[o.i];
      s.count[sl] += 1;
      out[o.j] = sl;
      order.push_back(sl);
    } else if (o.op == OWL_EDIT_DEL) {
      order.push_back(s.order[o.i]);
    } else {
      const uint32_t sl = (uint32_t)s.kid.size();
      s.kid.push_back(kids[o.j]);
      s.count.push_back(1);
      out[o.j] = sl;
      order.push_back(sl);
    }
  }
  s.order.swap(order);
  s.n_runs += 1;
  return out;
}

struct PlannedSeg {
  owl_segment s;
  uint32_t slot;
};

/* Gathers runs, checks classes, assigns slots.  Runs must be ascending and above `after`. */
owl_status plan_runs(owl_ctx* ctx, const uint32_t* runs, size_t n_runs, int64_t after, uint32_t* cls_io,
                     bool cls_known, SlotState& ss, std::vector<PlannedSeg>& plan) {
  std::vector<uint32_t> rs(runs, runs + n_runs);
  std::sort(rs.begin(), rs.end());
  for (size_t i = 1; i < rs.size(); ++i)
    if (rs[i] == rs[i - 1]) return fail(OWL_ERR_INVALID_ARG, "run %u listed twice", rs[i]);
  if (!rs.empty() && (int64_t)rs[0] <= after)
    return fail(OWL_ERR_INVALID_ARG, "run %u is not above the runs already merged (%lld)", rs[0], (long long)after);
  for (uint32_t r : rs) {
    auto lo = ctx->segs.lower_bound({r, 0});
    std::vector<uint32_t> seqs;
    std::vector<uint64_t> kids;
    std::vector<const owl_segment*> local;
    uint32_t cls = 0;
    bool have = false;
    for (auto it = lo; it != ctx->segs.end() && it->first.first == r; ++it) {
      seqs.push_back(it->first.second);
      kids.push_back(it->second.kernel_id);
      local.push_back(&it->second);
      cls = it->second.input_class;
      have = true;
    }
    if (!have) {
      auto rm = ctx->remote.find(r);
      if (rm == ctx->remote.end()) return fail(OWL_ERR_STATE, "run %u has not been ingested", r);
      cls = rm->second.cls;
      kids = rm->second.kids;
      for (size_t q = 0; q < kids.size(); ++q) seqs.push_back((uint32_t)q);
    }
    if (!cls_known) { *cls_io = cls; cls_known = true; }
    if (cls != *cls_io)
      return fail(OWL_ERR_INVALID_ARG, "run %u has input class %u, expected %u (one class per evidence)", r, cls, *cls_io);
    std::vector<uint32_t> sl = slot_merge(ss, seqs, kids);
    for (size_t q = 0; q < local.size(); ++q) plan.push_back({*local[q], sl[q]});
  }
  if (ss.kid.size() > OWL_MAX_SLOT)
    return fail(OWL_ERR_CAPACITY, "%zu evidence slots exceed the limit %u", ss.kid.size(), OWL_MAX_SLOT);
  return OWL_OK;
}

const char* kerr_text(uint32_t code) {
  switch (code) {
    case KERR_GWARP: return "gwarp >= n_warps";
    case KERR_BBFIELDS: return "non-zero addr/lane/ins on a BB_ENTRY";
    case KERR_MTYPE: return "unknown memory type";
    case KERR_NOBB: return "MEM record before the warp's first BB_ENTRY";
    case KERR_BBMISMATCH: return "MEM record bb != the warp's current BB";
    default: return "?";
  }
}

/* One fold pass over the planned segments into `tab` (A1-A3).  Returns OWL_OK, or an error; sets
   *overflow to the bitmask of tables that must grow.

   Device-resident segments are folded in one launch.  Host segments (OWL_SEG_HOST_RECORDS) are staged in waves
   of at most host_chunk_bytes (a wave holds at least one segment) through two device buffers: the copy of wave
   k + 1 (copy stream) overlaps the fold of wave k (context stream), and a buffer is refilled only after the fold
   that read it.  The channel-order segments of each launch are bucketed by warp on the device first, together
   and by bursts (their bytes again + 9 B per burst of scratch, held until the pass returns: the error report of
   a malformed record maps it back to the caller's order through its burst). */
owl_status fold_pass(owl_ctx* ctx, const std::vector<PlannedSeg>& plan, DevTable* tab, unsigned* overflow,
                     uint64_t* n_records) {
  const cudaStream_t st = ctx->stream;
  *overflow = 0;
  const uint32_t tile_shift = getenv("OWL_TILE_SHIFT") ? (uint32_t)atoi(getenv("OWL_TILE_SHIFT")) : 15u; /* tile sweep: profiles/r01_v4_ab.txt */
  std::vector<FoldSeg> fs(plan.size());
  std::vector<FoldBurst> fb(plan.size(), FoldBurst{nullptr, nullptr, nullptr, 0}); /* in-place channel order */
  std::vector<void*> scratch;
  std::vector<BucketedSet> sets; /* channel-order segments, bucketed per launch */
  std::vector<std::pair<uint32_t, uint32_t>> bucketed(plan.size(), {~0u, 0u}); /* (set, position) */
  uint64_t seen_words = 0, nrec = 0;
  for (size_t i = 0; i < plan.size(); ++i) seen_words += (plan[i].s.n_warps + 31) / 32;
  uint32_t* seen = (uint32_t*)owl_dev_alloc((seen_words + 1) * 4);
  if (!seen) return fail(OWL_ERR_OUT_OF_MEMORY, "fold: warp bitmap");
  scratch.push_back(seen);
  CUDA_TRY(cudaMemsetAsync(seen, 0, (seen_words + 1) * 4, st), "fold: memset");
  unsigned long long* walked = (unsigned long long*)owl_dev_alloc((plan.size() + 1) * 8);
  if (!walked) { owl_dev_free(seen); return fail(OWL_ERR_OUT_OF_MEMORY, "fold: walk counters"); }
  scratch.push_back(walked);
  CUDA_TRY(cudaMemsetAsync(walked, 0, (plan.size() + 1) * 8, st), "fold: memset");
  /* launches: device segments, then waves of host segments */
  const uint64_t chunk = ctx->cfg.host_chunk_bytes ? ctx->cfg.host_chunk_bytes : (256ull << 20);
  std::vector<std::vector<size_t>> launches(1);
  std::vector<uint64_t> wave_bytes(1, 0);
  for (size_t i = 0, so = 0; i < plan.size(); ++i) {
    const owl_segment& s = plan[i].s;
    fs[i].rec = (const uint4*)s.records;
    fs[i].n = s.n_records;
    fs[i].tile0 = 0;
    fs[i].slot = plan[i].slot;
    fs[i].n_warps = s.n_warps;
    fs[i].seen = seen + so;
    fs[i].walked = walked + i;
    fs[i].seg_index = (uint32_t)i;
    fs[i]._pad = 0;
    so += (s.n_warps + 31) / 32;
    nrec += s.n_records;
    if (!(s.flags & OWL_SEG_HOST_RECORDS) || !s.n_records) {
      launches[0].push_back(i);
      continue;
    }
    const uint64_t b = s.n_records * 16;
    if (launches.size() == 1 || (wave_bytes.back() && wave_bytes.back() + b > chunk)) {
      launches.emplace_back();
      wave_bytes.push_back(0);
    }
    launches.back().push_back(i);
    wave_bytes.back() += b;
  }
  uint64_t stage_cap = 0;
  for (size_t w = 1; w < wave_bytes.size(); ++w) stage_cap = std::max(stage_cap, wave_bytes[w]);
  uint4* stage[2] = {nullptr, nullptr};
  cudaEvent_t ready[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr};
  owl_status status = OWL_OK;
  if (stage_cap) {
    for (int k = 0; k < 2 && k + 1 < (int)launches.size(); ++k) {
      stage[k] = (uint4*)owl_dev_alloc(stage_cap);
      if (!stage[k]) status = fail(OWL_ERR_OUT_OF_MEMORY, "fold: host staging buffers (2 x %llu bytes)",
                                   (unsigned long long)stage_cap);
      else scratch.push_back(stage[k]);
      cudaEventCreateWithFlags(&ready[k], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&freed[k], cudaEventDisableTiming);
    }
    if (!ctx->copy_stream) cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking);
  }
  const int per_sm = ctx->cfg.fold_ctas_per_sm ? (int)ctx->cfg.fold_ctas_per_sm : owl_fold_ctas_per_sm();
  const int grid = ctx->n_sm * per_sm;
  uint32_t* vmap = status == OWL_OK ? (uint32_t*)owl_dev_alloc(owl_fold_scratch_bytes(grid)) : nullptr;
  if (status == OWL_OK && !vmap) status = fail(OWL_ERR_OUT_OF_MEMORY, "fold: visit-map scratch");
  if (vmap) scratch.push_back(vmap);
  FoldStatus hs;
  hs.first_error = ~0ull;
  hs.not_warp_major = ~0ull;
  hs.overflow = 0;
  hs.limit = 0;
  hs.tile_counter = 0;
  hs.n_flush = hs.n_bypass = hs.n_claim = 0;
  for (int i = 0; i < 8; ++i) hs.dbg[i] = 0;
  if (status == OWL_OK) cudaMemcpyAsync(ctx->d_status, &hs, sizeof hs, cudaMemcpyHostToDevice, st);
  std::vector<unsigned long long> walked_h(plan.size(), 0);
  float fold_ms = 0;
  uint64_t launched = 0;
  auto stage_wave = [&](size_t w) -> cudaError_t { /* copy stream: wave w into stage[(w - 1) % 2] */
    const int k = (int)((w - 1) & 1);
    cudaError_t e = cudaStreamWaitEvent(ctx->copy_stream, freed[k], 0);
    uint64_t off = 0;
    for (size_t i : launches[w]) {
      const owl_segment& s = plan[i].s;
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(stage[k] + off, s.records, s.n_records * 16, cudaMemcpyHostToDevice, ctx->copy_stream);
      fs[i].rec = stage[k] + off;
      off += s.n_records;
    }
    if (e == cudaSuccess) e = cudaEventRecord(ready[k], ctx->copy_stream);
    return e;
  };
  for (int k = 0; k < 2; ++k)
    if (freed[k]) cudaEventRecord(freed[k], st);
  if (status == OWL_OK && launches.size() > 1) {
    const cudaError_t e = stage_wave(1);
    if (e != cudaSuccess) status = cuda_fail(e, "fold: H2D staging");
  }
  for (size_t w = 0; w < launches.size() && status == OWL_OK; ++w) {
    if (w + 1 < launches.size() && w >= 1) { /* prefetch the next wave while this one is folded */
      const cudaError_t e = stage_wave(w + 1);
      if (e != cudaSuccess) { status = cuda_fail(e, "fold: H2D staging"); break; }
    }
    if (w >= 1) cudaStreamWaitEvent(st, ready[(w - 1) & 1], 0);
    { /* channel order: the launch's segments bucketed by warp together, by bursts (R17, N2) */
      std::vector<const uint4*> brec;
      std::vector<uint64_t> bn;
      std::vector<uint32_t> bw;
      std::vector<size_t> bi;
      for (size_t i : launches[w]) {
        const owl_segment& s = plan[i].s;
        if (!s.n_records || (s.flags & OWL_SEG_WARP_MAJOR)) continue;
        brec.push_back(fs[i].rec);
        bn.push_back(s.n_records);
        bw.push_back(s.n_warps);
        bi.push_back(i);
      }
      if (!bi.empty()) {
        /* walk the burst index in place (no 16 B per record of scratch; as fast as the copy for a tracer's bursts,
           profiles/r02_fold_experiments.txt #27) or copy to a warp-major buffer: owl_config.channel_order; AUTO
           folds in place whenever every segment has fewer than 2^32 records */
        bool fits = true;
        for (uint64_t x : bn) fits = fits && x < (1ull << 32);
        /* host-record waves (w >= 1) are copied: their staging buffers are reused by later waves, and a malformed
           record's report re-reads the bucketed records after the last wave */
        const bool inplace = ctx->cfg.channel_order != OWL_CHANNEL_COPY && fits && w == 0;
        sets.emplace_back();
        const auto tb0 = std::chrono::steady_clock::now();
        const cudaError_t e = owl_bucket_segments(brec, bn, bw, &sets.back(), st, !inplace);
        if (getenv("OWL_FOLD_VERBOSE"))
          fprintf(stderr, "[owl] bucketing %s: %.3f ms (host, synchronous)\n", inplace ? "in place" : "copy",
                  std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tb0).count());
        if (e != cudaSuccess) { status = cuda_fail(e, "fold: bucketing"); break; }
        const BucketedSet& bs = sets.back();
        for (size_t k = 0; k < bi.size(); ++k) {
          if (inplace) {
            FoldBurst& f = fb[bi[k]];
            f.bvs = bs.bvs + bs.bfirst[k];
            f.bpo = bs.bpo + bs.bfirst[k];
            f.bk = bs.bk + bs.bfirst[k];
            f.nb = bs.bfirst[k + 1] - bs.bfirst[k];
          } else {
            fs[bi[k]].rec = bs.out + bs.off[k];
          }
          bucketed[bi[k]] = {(uint32_t)sets.size() - 1, (uint32_t)k};
        }
      }
    }
    /* work items: (segment, tile of 2^tile_shift records), one range per segment; in-place channel-order segments
       (bursts walked through their index) get their own launch of fold_burst_kernel, items of 2^burst_shift bursts */
    const uint32_t burst_shift = getenv("OWL_BURST_SHIFT") ? (uint32_t)atoi(getenv("OWL_BURST_SHIFT")) : 10u;
    cudaError_t e = cudaSuccess;
    bool any = false;
    for (int mode = 0; mode < 2 && e == cudaSuccess; ++mode) {
      std::vector<FoldSeg> lsegs;
      std::vector<FoldBurst> lbursts;
      std::vector<FoldGroup> groups;
      uint64_t items = 0;
      const uint32_t shift = mode ? burst_shift : tile_shift;
      for (size_t i : launches[w]) {
        if ((fb[i].bvs != nullptr) != (mode == 1)) continue;
        const uint64_t units = mode ? fb[i].nb : fs[i].n;
        const uint64_t ntile = (units + (1ull << shift) - 1) >> shift;
        if (!ntile) continue;
        FoldGroup g;
        g.item0 = items;
        g.first_seg = (uint32_t)lsegs.size();
        g._pad = 0;
        lsegs.push_back(fs[i]);
        lbursts.push_back(fb[i]);
        groups.push_back(g);
        items += ntile;
      }
      if (!items) continue;
      FoldBurst* dbursts = nullptr;
      if (mode) {
        dbursts = (FoldBurst*)owl_dev_alloc(lbursts.size() * sizeof(FoldBurst) + 16);
        if (!dbursts) { e = cudaErrorMemoryAllocation; break; }
        scratch.push_back(dbursts);
        cudaMemcpyAsync(dbursts, lbursts.data(), lbursts.size() * sizeof(FoldBurst), cudaMemcpyHostToDevice, st);
      }
      FoldSeg* dsegs = (FoldSeg*)owl_dev_alloc(lsegs.size() * sizeof(FoldSeg) + 16);
      FoldGroup* dgroups = (FoldGroup*)owl_dev_alloc(groups.size() * sizeof(FoldGroup) + 16);
      if (!dsegs || !dgroups) { owl_dev_free(dsegs); owl_dev_free(dgroups); e = cudaErrorMemoryAllocation; break; }
      scratch.push_back(dsegs);
      scratch.push_back(dgroups);
      cudaMemcpyAsync(dsegs, lsegs.data(), lsegs.size() * sizeof(FoldSeg), cudaMemcpyHostToDevice, st);
      cudaMemcpyAsync(dgroups, groups.data(), groups.size() * sizeof(FoldGroup), cudaMemcpyHostToDevice, st);
      cudaMemsetAsync(&ctx->d_status->tile_counter, 0, sizeof(unsigned long long), st); /* the launch's work counter */
      FoldArgs a;
      a.segs = dsegs;
      a.groups = dgroups;
      a.n_groups = (uint32_t)groups.size();
      a.tile_shift = shift;
      a.n_items = items;
      for (int t = 0; t < T_NUM; ++t) a.tab[t] = tab[t];
      a.status = ctx->d_status;
      a.mode = getenv("OWL_FOLD_MODE") ? (uint32_t)atoi(getenv("OWL_FOLD_MODE")) : 0u;
      a.vmap = vmap;
      if (!any) cudaEventRecord(ctx->ev0, st);
      any = true;
      e = mode ? owl_launch_fold_bursts(a, dbursts, grid, st) : owl_launch_fold(a, grid, st);
    }
    if (!any && e == cudaSuccess) {
      if (w >= 1) cudaEventRecord(freed[(w - 1) & 1], st);
      continue;
    }
    cudaEventRecord(ctx->ev1, st);
    if (w >= 1) cudaEventRecord(freed[(w - 1) & 1], st);
    if (e == cudaSuccess && launches.size() > 1) e = cudaEventSynchronize(ctx->ev1); /* per-launch timing */
    if (e != cudaSuccess) { status = cuda_fail(e, "fold kernel"); break; }
    if (launches.size() > 1) {
      float ms = 0;
      cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1);
      fold_ms += ms;
    }
    ++launched;
  }
  cudaError_t e = status == OWL_OK ? cudaMemcpyAsync(&hs, ctx->d_status, sizeof hs, cudaMemcpyDeviceToHost, st)
                                   : cudaSuccess;
  if (status == OWL_OK && e == cudaSuccess)
    e = cudaMemcpyAsync(walked_h.data(), walked, plan.size() * 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (ctx->copy_stream) cudaStreamSynchronize(ctx->copy_stream);
  for (int k = 0; k < 2; ++k) {
    if (ready[k]) cudaEventDestroy(ready[k]);
    if (freed[k]) cudaEventDestroy(freed[k]);
  }
  if (status == OWL_OK && e != cudaSuccess) status = cuda_fail(e, "fold kernel");
  if (status == OWL_OK) {
    if (launches.size() == 1) {
      float ms = 0;
      if (launched) cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1);
      fold_ms = ms;
    }
    ctx->fold_launches += launched;
    ctx->last_fold_ms = fold_ms;
    ctx->last_fold_records = nrec;
    ctx->total_fold_ms += fold_ms;
    ctx->total_fold_records += nrec;
    if (getenv("OWL_FOLD_VERBOSE")) {
      fprintf(stderr, "[owl] fold: %llu records %.3f ms pages %llu page-adds %llu claims %llu (%llu launches)\n",
              (unsigned long long)nrec, fold_ms, hs.n_flush, hs.n_bypass, hs.n_claim, (unsigned long long)launched);
      if (hs.dbg[0] | hs.dbg[1])
        fprintf(stderr, "[owl] fold stats: fast %llu slow %llu %llu %llu %llu %llu %llu %llu\n", hs.dbg[0],
                hs.dbg[1], hs.dbg[2], hs.dbg[3], hs.dbg[4], hs.dbg[5], hs.dbg[6], hs.dbg[7]);
    }
  }
  if (status == OWL_OK) {
    /* An overflowed pass stopped early: its reports are incomplete, the regrown pass decides.  A segment that
       is flagged warp-major but is not (a warp seen twice, or records the warp walk did not cover exactly once)
       is reported first: walking it from the middle of a warp produces malformed-record artifacts. */
    /* (bucketed channel-order segments are warp-major by construction: a walk mismatch there comes from records
       with out-of-range gwarps, which a malformed-record report already covers) */
    const bool reported = hs.first_error != ~0ull;
    size_t bad_walk = plan.size();
    for (size_t i = 0; i < plan.size() && bad_walk == plan.size(); ++i)
      if (walked_h[i] != plan[i].s.n_records && !(reported && bucketed[i].first != ~0u)) bad_walk = i;
    const uint32_t nwm_seg = (uint32_t)(hs.not_warp_major >> 32);
    if (hs.overflow) {
    } else if (hs.not_warp_major != ~0ull && !(reported && nwm_seg < plan.size() && bucketed[nwm_seg].first != ~0u)) {
      const uint32_t si = (uint32_t)(hs.not_warp_major >> 32);
      status = fail(OWL_ERR_INVALID_ARG,
                    "segment (run %u, seq %u) is flagged OWL_SEG_WARP_MAJOR but warp %u's records are not contiguous",
                    plan[si].s.run, plan[si].s.seq, (uint32_t)hs.not_warp_major);
    } else if (bad_walk < plan.size()) {
      const size_t si = bad_walk;
      status = fail(OWL_ERR_INVALID_ARG,
                    "segment (run %u, seq %u) is flagged OWL_SEG_WARP_MAJOR but its records are not grouped by warp "
                    "(the warp walk covered %llu records of %llu)",
                    plan[si].s.run, plan[si].s.seq, (unsigned long long)walked_h[si],
                    (unsigned long long)plan[si].s.n_records);
    } else if (hs.first_error != ~0ull) {
      const uint32_t si = (uint32_t)(hs.first_error >> 40);
      uint64_t idx = (hs.first_error >> 3) & ((1ull << 37) - 1);
      uint32_t code = (uint32_t)(hs.first_error & 7);
      if (si < plan.size() && bucketed[si].first != ~0u) { /* bucketed: the first bad record in the caller's order */
        unsigned long long ic = ~0ull;
        const cudaError_t e = owl_first_bad_record(sets[bucketed[si].first], bucketed[si].second, plan[si].s.n_warps,
                                                   &ic, st);
        if (e == cudaSuccess && ic != ~0ull) {
          idx = ic >> 3;
          code = (uint32_t)(ic & 7);
        }
      }
      status = fail(OWL_ERR_MALFORMED_TRACE, "malformed trace: run %u seq %u record %llu: %s",
                    si < plan.size() ? plan[si].s.run : 0, si < plan.size() ? plan[si].s.seq : 0,
                    (unsigned long long)idx, kerr_text(code));
    } else if (hs.limit) {
      status = (hs.limit & 2) ? fail(OWL_ERR_CAPACITY, "a traced warp visits more than %d distinct basic blocks",
                                     owl_fold_max_bbs())
                              : fail(OWL_ERR_CAPACITY, "a basic-block visit ordinal j exceeds 2^22-1");
    }
    *overflow = hs.overflow;
  }
  for (void* p : scratch) owl_dev_free(p);
  for (BucketedSet& b : sets) owl_bucketed_free(&b);
  *n_records = nrec;
  return status;
}

uint64_t default_cap(owl_ctx* ctx, int t) {
  if (ctx->cap_hint[t]) return ctx->cap_hint[t];
  if (t == T_ADDR) return ctx->cfg.addr_capacity ? next_pow2(ctx->cfg.addr_capacity) : (1ull << 20);
  return ctx->cfg.cf_capacity ? next_pow2(ctx->cfg.cf_capacity) : (1ull << 14);
}

/* Builds fresh tables for the planned segments, regrowing on overflow. */
owl_status build_tables(owl_ctx* ctx, const std::vector<PlannedSeg>& plan, DevTable* tab, uint64_t* n_records) {
  uint64_t cap[T_NUM];
  for (int t = 0; t < T_NUM; ++t) cap[t] = default_cap(ctx, t);
  const uint32_t max_regrow = ctx->cfg.max_regrow ? ctx->cfg.max_regrow : 6;
  for (uint32_t attempt = 0;; ++attempt) {
    for (int t = 0; t < T_NUM; ++t) {
      cudaError_t e = owl_table_alloc(&tab[t], cap[t], ctx->stream);
      if (e != cudaSuccess) {
        for (int u = 0; u <= t; ++u) owl_table_free(&tab[u]);
        return cuda_fail(e, "table allocation");
      }
    }
    unsigned overflow = 0;
    owl_status s = fold_pass(ctx, plan, tab, &overflow, n_records);
    if (s != OWL_OK) {
      for (int t = 0; t < T_NUM; ++t) owl_table_free(&tab[t]);
      return s;
    }
    if (!overflow) {
      /* next builds: at most 1/8 of the address cells claimed (load shift 3, profiles/r01_v4_ab.txt), so nearly every key sits in its home
         bucket and the fold's first probe hits (owl_fold.cu) */
      unsigned long long fill = 0;
      cudaMemcpy(&fill, tab[T_ADDR].fill, sizeof fill, cudaMemcpyDeviceToHost);
      static const int load_shift = getenv("OWL_ADDR_LOAD_SHIFT") ? atoi(getenv("OWL_ADDR_LOAD_SHIFT")) : 3;
      ctx->cap_hint[T_ADDR] = std::max(ctx->cap_hint[T_ADDR], std::min<uint64_t>(next_pow2(fill << load_shift), 1ull << 28));
      for (int t = 0; t < T_NUM; ++t) ctx->cap_hint[t] = std::max(ctx->cap_hint[t], cap[t]);
      return OWL_OK;
    }
    for (int t = 0; t < T_NUM; ++t) owl_table_free(&tab[t]);
    if (attempt >= max_regrow) return fail(OWL_ERR_CAPACITY, "A-DCFG tables still full after %u regrowths", attempt);
    for (int t = 0; t < T_NUM; ++t)
      if (overflow & (1u << t)) cap[t] *= 4;
  }
}

owl_status ensure_sorted(owl_adcfg* g) {
  if (g->sorted_ok) return OWL_OK;
  for (int t = 0; t < T_NUM; ++t) owl_sorted_free(&g->sorted[t]);
  cudaError_t e = owl_tables_sorted(g->tab, T_NUM, g->sorted, g->ctx->stream);
  if (e != cudaSuccess) return cuda_fail(e, "canonical sort");
  g->sorted_ok = true;
  return OWL_OK;
}

/* Merges the cells of `src` (sorted) into g's tables, rebuilding them with room for both. */
owl_status merge_into(owl_adcfg* g, SortedTable* src) {
  owl_status s = ensure_sorted(g);
  if (s != OWL_OK) return s;
  cudaStream_t st = g->ctx->stream;
  for (int t = 0; t < T_NUM; ++t) {
    const uint64_t need = g->sorted[t].n + src[t].n;
    uint64_t cap = std::max<uint64_t>(g->tab[t].cap, next_pow2(2 * need + 16));
    DevTable nt{};
    CUDA_TRY(owl_table_alloc(&nt, cap, st), "merge: table allocation");
    CUDA_TRY(cudaMemsetAsync(g->ctx->d_status, 0, sizeof(FoldStatus), st), "merge");
    CUDA_TRY(owl_table_insert_sorted(nt, t, g->sorted[t].k, g->sorted[t].c, g->sorted[t].n, g->ctx->d_status, st), "merge");
    CUDA_TRY(owl_table_insert_sorted(nt, t, src[t].k, src[t].c, src[t].n, g->ctx->d_status, st), "merge");
    CUDA_TRY(cudaStreamSynchronize(st), "merge");
    owl_table_free(&g->tab[t]);
    g->tab[t] = nt;
  }
  g->sorted_ok = false;
  return OWL_OK;
}

template <class T>
T* host_copy(const std::vector<T>& v) {
  T* p = (T*)malloc(sizeof(T) * (v.size() ? v.size() : 1));
  if (p && !v.empty()) memcpy(p, v.data(), sizeof(T) * v.size());
  return p;
}

/* unpack canonical keys into row fields */
void unpack(int t, const Key128& k, uint32_t& slot, uint32_t& a, uint32_t& b, uint32_t& c, uint64_t& x) {
  if (t == T_ADDR) {
    slot = (uint32_t)(k.hi >> 48);
    a = (uint32_t)((k.hi >> 30) & 0x3FFFFu); /* bb */
    b = (uint32_t)((k.hi >> 22) & 0xFFu);    /* ins */
    c = (uint32_t)(k.hi & OWL_MAX_J);        /* j */
    x = k.lo;
  } else {
    slot = (uint32_t)(k.hi >> 32);
    a = (uint32_t)k.hi; /* bb or src */
    b = (uint32_t)(k.lo >> 32);
    c = (uint32_t)k.lo;
    x = 0;
  }
}

}  // namespace

/* ================================== ABI ================================== */

OWL_API const char* owl_last_error(void) { return g_err.c_str(); }
OWL_API const char* owl_version(void) { return "owl-b200 0.1 (sm_100a)"; }
OWL_API void owl_free(void* p) { owl_host_free(p); }

OWL_API owl_status owl_ctx_create(int cuda_device, owl_ctx** out) {
  if (!out) return fail(OWL_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0) return fail(OWL_ERR_CUDA, "no CUDA device: %s", cudaGetErrorString(e));
  if (cuda_device < 0 || cuda_device >= n) return fail(OWL_ERR_INVALID_ARG, "device %d out of range", cuda_device);
  CUDA_TRY(cudaSetDevice(cuda_device), "cudaSetDevice");
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, cuda_device), "cudaGetDeviceProperties");
  if (prop.major < 10) return fail(OWL_ERR_CUDA, "device %d is sm_%d%d; libowl is built for sm_100a", cuda_device, prop.major, prop.minor);
  owl_ctx* c = new owl_ctx();
  c->device = cuda_device;
  c->n_sm = prop.multiProcessorCount;
  c->d_status = (FoldStatus*)owl_dev_alloc(sizeof(FoldStatus));
  if (!c->d_status) { delete c; return fail(OWL_ERR_OUT_OF_MEMORY, "status"); }
  cudaEventCreate(&c->ev0);
  cudaEventCreate(&c->ev1);
  *out = c;
  return OWL_OK;
}

OWL_API owl_status owl_ctx_destroy(owl_ctx* ctx) {
  if (!ctx) return OWL_OK;
  cudaSetDevice(ctx->device);
  owl_dev_free(ctx->d_status);
  owl_dev_trim(ctx->device);
  if (ctx->ev0) cudaEventDestroy(ctx->ev0);
  if (ctx->ev1) cudaEventDestroy(ctx->ev1);
  if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
  delete ctx;
  return OWL_OK;
}

OWL_API owl_status owl_ctx_set_config(owl_ctx* ctx, const owl_config* cfg) {
  if (!ctx) return fail(OWL_ERR_INVALID_ARG, "ctx is NULL");
  if (cfg && cfg->hcf_reading > OWL_HCF_ROW_NORMALIZED)
    return fail(OWL_ERR_INVALID_ARG, "hcf_reading must be OWL_HCF_COUNTS or OWL_HCF_ROW_NORMALIZED");
  if (cfg && cfg->channel_order > OWL_CHANNEL_IN_PLACE)
    return fail(OWL_ERR_INVALID_ARG, "channel_order must be OWL_CHANNEL_AUTO, OWL_CHANNEL_COPY or OWL_CHANNEL_IN_PLACE");
  if (cfg) ctx->cfg = *cfg;
  else ctx->cfg = owl_config{};
  for (int t = 0; t < T_NUM; ++t) ctx->cap_hint[t] = 0;
  return OWL_OK;
}

OWL_API owl_status owl_ingest_traces(owl_ctx* ctx, const owl_segment* segs, size_t n_segs, owl_stream_t stream) {
  OWL_RANGE();
  if (!ctx || (!segs && n_segs)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  for (size_t i = 0; i < n_segs; ++i) {
    const owl_segment& s = segs[i];
    if (s.n_records && !s.records) return fail(OWL_ERR_INVALID_ARG, "segment %zu: records is NULL", i);
    if (s.input_class > 1) return fail(OWL_ERR_INVALID_ARG, "segment %zu: input_class %u", i, s.input_class);
    if (((uintptr_t)s.records & 15) != 0) return fail(OWL_ERR_INVALID_ARG, "segment %zu: records not 16-byte aligned", i);
    if (ctx->segs.count({s.run, s.seq})) return fail(OWL_ERR_INVALID_ARG, "segment (run %u, seq %u) already ingested", s.run, s.seq);
    auto lo = ctx->segs.lower_bound({s.run, 0});
    if (lo != ctx->segs.end() && lo->first.first == s.run && lo->second.input_class != s.input_class)
      return fail(OWL_ERR_INVALID_ARG, "run %u: segments of different input classes", s.run);
    for (size_t j = 0; j < i; ++j)
      if (segs[j].run == s.run && segs[j].seq == s.seq) return fail(OWL_ERR_INVALID_ARG, "segment (run %u, seq %u) twice", s.run, s.seq);
  }
  for (size_t i = 0; i < n_segs; ++i) ctx->segs[{segs[i].run, segs[i].seq}] = segs[i];
  ctx->stream = (cudaStream_t)stream;
  return OWL_OK;
}

OWL_API owl_status owl_forget_runs(owl_ctx* ctx, const uint32_t* runs, size_t n_runs) {
  if (!ctx || (!runs && n_runs)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  for (size_t i = 0; i < n_runs; ++i) {
    auto lo = ctx->segs.lower_bound({runs[i], 0});
    while (lo != ctx->segs.end() && lo->first.first == runs[i]) lo = ctx->segs.erase(lo);
    ctx->remote.erase(runs[i]);
  }
  return OWL_OK;
}

OWL_API owl_status owl_register_remote_runs(owl_ctx* ctx, const uint32_t* runs, const uint32_t* classes,
                                            const uint32_t* seq_len, const uint64_t* kernel_ids, size_t n_runs) {
  if (!ctx || (n_runs && (!runs || !classes || !seq_len))) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  size_t off = 0;
  for (size_t i = 0; i < n_runs; ++i) {
    RemoteRun rr;
    rr.cls = classes[i];
    rr.kids.assign(kernel_ids + off, kernel_ids + off + seq_len[i]);
    off += seq_len[i];
    ctx->remote[runs[i]] = rr;
  }
  return OWL_OK;
}

OWL_API owl_status owl_build_adcfg(owl_ctx* ctx, const uint32_t* runs, size_t n_runs, owl_adcfg** out) {
  OWL_RANGE();
  if (!ctx || !out || (!runs && n_runs)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  *out = nullptr;
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  owl_adcfg* g = new owl_adcfg();
  g->ctx = ctx;
  std::vector<PlannedSeg> plan;
  owl_status s = plan_runs(ctx, runs, n_runs, -1, &g->cls, false, g->slots, plan);
  if (s == OWL_OK) s = build_tables(ctx, plan, g->tab, &g->n_records);
  if (s != OWL_OK) { delete g; return s; }
  for (size_t i = 0; i < n_runs; ++i) g->max_run = std::max<int64_t>(g->max_run, runs[i]);
  *out = g;
  return OWL_OK;
}

OWL_API owl_status owl_adcfg_accumulate(owl_ctx* ctx, owl_adcfg* g, const uint32_t* runs, size_t n_runs) {
  OWL_RANGE();
  if (!ctx || !g || (!runs && n_runs)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  if (!n_runs) return OWL_OK;
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  SlotState ss = g->slots;
  std::vector<PlannedSeg> plan;
  uint32_t cls = g->cls;
  owl_status s = plan_runs(ctx, runs, n_runs, g->max_run, &cls, g->slots.n_runs > 0, ss, plan);
  if (s != OWL_OK) return s;
  owl_adcfg tmp;
  tmp.ctx = ctx;
  uint64_t nrec = 0;
  s = build_tables(ctx, plan, tmp.tab, &nrec);
  if (s == OWL_OK) s = ensure_sorted(&tmp);
  if (s == OWL_OK) s = merge_into(g, tmp.sorted);
  if (s != OWL_OK) return s;
  g->slots = ss;
  g->cls = cls;
  g->n_records += nrec;
  for (size_t i = 0; i < n_runs; ++i) g->max_run = std::max<int64_t>(g->max_run, runs[i]);
  return OWL_OK;
}

OWL_API owl_status owl_adcfg_info_get(const owl_adcfg* g, owl_adcfg_info* info) {
  if (!g || !info) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  owl_status s = ensure_sorted(const_cast<owl_adcfg*>(g));
  if (s != OWL_OK) return s;
  info->input_class = g->cls;
  info->n_runs = g->slots.n_runs;
  info->n_slots = (uint32_t)g->slots.order.size();
  info->_pad = 0;
  for (int t = 0; t < T_NUM; ++t) info->n_cells[t] = g->sorted[t].n;
  info->n_records = g->n_records;
  return OWL_OK;
}

OWL_API owl_status owl_adcfg_destroy(owl_adcfg* g) {
  if (g) {
    cudaSetDevice(g->ctx->device);
    delete g;
  }
  return OWL_OK;
}

OWL_API owl_status owl_adcfg_export(const owl_adcfg* gc, const char* path, void** host_blob, size_t* bytes) {
  OWL_RANGE();
  if (!gc) return fail(OWL_ERR_INVALID_ARG, "NULL adcfg");
  owl_adcfg* g = const_cast<owl_adcfg*>(gc);
  CUDA_TRY(cudaSetDevice(g->ctx->device), "cudaSetDevice");
  owl_status s = ensure_sorted(g);
  if (s != OWL_OK) return s;
  std::vector<Key128> k[T_NUM];
  std::vector<unsigned long long> c[T_NUM];
  for (int t = 0; t < T_NUM; ++t) {
    k[t].resize(g->sorted[t].n);
    c[t].resize(g->sorted[t].n);
    if (g->sorted[t].n) {
      CUDA_TRY(cudaMemcpy(k[t].data(), g->sorted[t].k, g->sorted[t].n * sizeof(Key128), cudaMemcpyDeviceToHost), "export");
      CUDA_TRY(cudaMemcpy(c[t].data(), g->sorted[t].c, g->sorted[t].n * 8, cudaMemcpyDeviceToHost), "export");
    }
  }
  std::vector<unsigned char> out;
  auto put = [&](const void* p, size_t n) { const unsigned char* q = (const unsigned char*)p; out.insert(out.end(), q, q + n); };
  auto u32 = [&](uint32_t v) { put(&v, 4); };
  auto u64 = [&](uint64_t v) { put(&v, 8); };
  size_t need = 56 + g->slots.order.size() * 24 + k[0].size() * 16 + k[1].size() * 24 + k[2].size() * 24 + k[3].size() * 32;
  out.reserve(need);
  put("OWLADCFG", 8);
  u32(1);
  u32(g->cls);
  u32(g->slots.n_runs);
  u32((uint32_t)g->slots.order.size());
  for (int t = 0; t < T_NUM; ++t) u64(k[t].size());
  for (uint32_t sl : g->slots.order) { u32(sl); u32(0); u64(g->slots.kid[sl]); u64(g->slots.count[sl]); }
  for (int t = 0; t < T_NUM; ++t)
    for (size_t i = 0; i < k[t].size(); ++i) {
      uint32_t slot, a, b, cc;
      uint64_t x;
      unpack(t, k[t][i], slot, a, b, cc, x);
      if (t == T_NODE) { u32(slot); u32(a); }
      else if (t == T_EDGE) { u32(slot); u32(a); u32(cc); u32(0); }
      else if (t == T_TRIPLE) { u32(slot); u32(a); u32(b); u32(cc); }
      else { u32(slot); u32(a); u32(b); u32(cc); u64(x); }
      u64(c[t][i]);
    }
  if (path) {
    FILE* f = fopen(path, "wb");
    if (!f) return fail(OWL_ERR_INVALID_ARG, "cannot open %s", path);
    size_t w = fwrite(out.data(), 1, out.size(), f);
    fclose(f);
    if (w != out.size()) return fail(OWL_ERR_INVALID_ARG, "short write to %s", path);
  }
  if (host_blob) {
    *host_blob = host_copy(out);
    if (!*host_blob) return fail(OWL_ERR_OUT_OF_MEMORY, "export blob");
  }
  if (bytes) *bytes = out.size();
  return OWL_OK;
}

OWL_API owl_status owl_diff_adcfg(owl_ctx* ctx, const owl_adcfg* a, const owl_adcfg* b, owl_diff** rows, size_t* n_rows) {
  OWL_RANGE();
  if (!ctx || !a || !b || !rows || !n_rows) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  owl_adcfg* ga = const_cast<owl_adcfg*>(a);
  owl_adcfg* gb = const_cast<owl_adcfg*>(b);
  static const bool verbose = getenv("OWL_DIFF_VERBOSE") != nullptr;
  auto now = [] { return std::chrono::steady_clock::now(); };
  auto t0 = now();
  owl_status s = ensure_sorted(ga);
  auto t1 = now();
  if (s == OWL_OK) s = ensure_sorted(gb);
  auto t2 = now();
  if (s != OWL_OK) return s;
  const uint32_t NA = 0xFFFFFFFFu;
  owl_diff* dev_rows = nullptr;
  uint64_t nd = 0;
  const size_t extra = ga->slots.order.size() + gb->slots.order.size();
  CUDA_TRY(owl_diff_rows(ga->sorted, gb->sorted, T_NUM, &dev_rows, &nd, extra, ctx->stream), "diff");
  auto t3 = now();
  if (verbose)
    fprintf(stderr, "[owl] diff: sort a %.3f ms, sort b %.3f ms, join + rows %.3f ms (%llu rows)\n",
            std::chrono::duration<double, std::milli>(t1 - t0).count(),
            std::chrono::duration<double, std::milli>(t2 - t1).count(),
            std::chrono::duration<double, std::milli>(t3 - t2).count(), (unsigned long long)nd);
  /* slot table: (slot, kernel_id) -> invocation count */
  std::map<std::pair<uint32_t, uint64_t>, uint64_t> sa, sb;
  for (uint32_t sl : ga->slots.order) sa[{sl, ga->slots.kid[sl]}] = ga->slots.count[sl];
  for (uint32_t sl : gb->slots.order) sb[{sl, gb->slots.kid[sl]}] = gb->slots.count[sl];
  std::map<std::pair<uint32_t, uint64_t>, std::pair<uint64_t, uint64_t>> all;
  for (auto& e : sa) all[e.first].first = e.second;
  for (auto& e : sb) all[e.first].second = e.second;
  for (auto& e : all)
    if (e.second.first != e.second.second) {
      owl_diff& r = dev_rows[nd++];
      r.table = OWL_TABLE_SLOT;
      r.slot = e.first.first;
      r.bb = r.ins = r.j = r.prev = r.next = NA;
      r._pad = 0;
      r.x = e.first.second;
      r.count_a = e.second.first;
      r.count_b = e.second.second;
    }
  *rows = dev_rows;
  *n_rows = nd;
  return OWL_OK;
}

namespace {

struct Alignment {
  std::vector<OwlEdit> ops;
  std::vector<uint32_t> f2r;   /* fix slot -> rnd slot (UINT32_MAX if unaligned) */
  std::vector<int> pos_of_f;   /* fix slot -> script position */
};

Alignment align(const owl_adcfg* f, const owl_adcfg* r) {
  Alignment al;
  std::vector<uint64_t> a, b;
  for (uint32_t s : f->slots.order) a.push_back(f->slots.kid[s]);
  for (uint32_t s : r->slots.order) b.push_back(r->slots.kid[s]);
  al.ops = owl_myers(a, b);
  al.f2r.assign(f->slots.kid.size(), 0xFFFFFFFFu);
  al.pos_of_f.assign(f->slots.kid.size(), -1);
  for (size_t p = 0; p < al.ops.size(); ++p)
    if (al.ops[p].op == OWL_EDIT_MATCH) {
      const uint32_t sf = f->slots.order[al.ops[p].i];
      al.f2r[sf] = r->slots.order[al.ops[p].j];
      al.pos_of_f[sf] = (int)p;
    }
  return al;
}

owl_status run_ks(owl_ctx* ctx, const owl_adcfg* f, const owl_adcfg* r, double sig, const Alignment& al,
                  std::vector<owl_ks_row>& rows, std::vector<int>& pos) {
  owl_status s = ensure_sorted(const_cast<owl_adcfg*>(f));
  if (s == OWL_OK) s = ensure_sorted(const_cast<owl_adcfg*>(r));
  if (s != OWL_OK) return s;
  const uint32_t NA = 0xFFFFFFFFu;
  std::vector<std::tuple<int, uint32_t, uint32_t, uint32_t, uint32_t, size_t>> order;
  for (int tbl : {T_TRIPLE, T_ADDR}) {
    std::vector<KsOutRow> out;
    CUDA_TRY(owl_ks_run(tbl, f->sorted[tbl], r->sorted[tbl], al.f2r, sig, (int)ctx->cfg.hcf_reading, out,
                        ctx->stream), "KS tests");
    for (const KsOutRow& o : out) {
      owl_ks_row row;
      Key128 kf{o.hi_f, 0}, kr{o.hi_r, 0};
      uint32_t sf, sr, a1, a2, a3, b1, b2, b3;
      uint64_t x;
      unpack(tbl, kf, sf, a1, a2, a3, x);
      unpack(tbl, kr, sr, b1, b2, b3, x);
      row.kind = tbl == T_TRIPLE ? OWL_LEAK_CONTROL_FLOW : OWL_LEAK_DATA_FLOW;
      row.slot_fix = sf;
      row.slot_rnd = sr;
      row.bb = a1;
      row.ins = tbl == T_ADDR ? a2 : NA;
      row.j = tbl == T_ADDR ? a3 : NA;
      row.n = o.n; row.m = o.m; row.K_lo = o.K_lo; row.K_hi = o.K_hi;
      row.D = o.D; row.p = o.p; row.fail = o.fail; row._pad = 0;
      order.emplace_back(al.pos_of_f[sf], row.kind, row.bb, row.ins, row.j, rows.size());
      rows.push_back(row);
    }
  }
  std::sort(order.begin(), order.end());
  std::vector<owl_ks_row> sorted;
  pos.clear();
  for (auto& o : order) { sorted.push_back(rows[std::get<5>(o)]); pos.push_back(std::get<0>(o)); }
  rows.swap(sorted);
  return OWL_OK;
}

}  // namespace

OWL_API owl_status owl_ks_tests(owl_ctx* ctx, const owl_adcfg* e_fix, const owl_adcfg* e_rnd, double significance,
                                owl_ks_row** rows, size_t* n_rows) {
  OWL_RANGE();
  if (!ctx || !e_fix || !e_rnd || !rows || !n_rows) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  Alignment al = align(e_fix, e_rnd);
  std::vector<owl_ks_row> out;
  std::vector<int> pos;
  owl_status s = run_ks(ctx, e_fix, e_rnd, significance, al, out, pos);
  if (s != OWL_OK) return s;
  *rows = host_copy(out);
  *n_rows = out.size();
  return OWL_OK;
}

/* N1 (§VI): partition runs by identical per-run A-DCFGs.  Fingerprints bucket, exact
   comparisons with each class's representative decide. */
OWL_API owl_status owl_filter_inputs(owl_ctx* ctx, const uint32_t* runs, size_t n_runs, uint32_t* class_of,
                                     uint32_t* n_classes) {
  OWL_RANGE();
  if (!ctx || !n_classes || (n_runs && (!runs || !class_of))) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  for (size_t i = 0; i < n_runs; ++i)
    for (size_t j = 0; j < i; ++j)
      if (runs[i] == runs[j]) return fail(OWL_ERR_INVALID_ARG, "run %u given twice", runs[i]);
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  struct Rep {
    std::unique_ptr<owl_adcfg> g;
    uint32_t cls;
  };
  std::map<std::pair<unsigned long long, unsigned long long>, std::vector<Rep>> buckets;
  uint32_t nc = 0;
  for (size_t i = 0; i < n_runs; ++i) {
    owl_adcfg* raw = nullptr;
    owl_status st = owl_build_adcfg(ctx, &runs[i], 1, &raw);
    if (st != OWL_OK) return st;
    std::unique_ptr<owl_adcfg> g(raw);
    st = ensure_sorted(g.get());
    if (st != OWL_OK) return st;
    for (int t = 0; t < T_NUM; ++t) owl_table_free(&g->tab[t]); /* only the sorted cells are compared */
    unsigned long long fp[2];
    CUDA_TRY(owl_tables_fingerprint(g->sorted, T_NUM, fp, ctx->stream), "filter: fingerprint");
    for (uint32_t sl : g->slots.order) { /* the kernel sequence is part of the trace */
      fp[0] = owl_mix64(fp[0] ^ g->slots.kid[sl]);
      fp[1] = owl_mix64(fp[1] + g->slots.kid[sl] * 0x9E3779B97F4A7C15ull + g->slots.count[sl]);
    }
    std::vector<Rep>& cand = buckets[{fp[0], fp[1]}];
    int found = -1;
    for (const Rep& r : cand) {
      const owl_adcfg* a = r.g.get();
      bool same = a->slots.order == g->slots.order && a->slots.kid == g->slots.kid && a->slots.count == g->slots.count;
      if (same) {
        owl_diff* rows = nullptr;
        uint64_t nd = 0;
        CUDA_TRY(owl_diff_rows(a->sorted, g->sorted, T_NUM, &rows, &nd, 0, ctx->stream), "filter: compare");
        owl_host_free(rows);
        same = nd == 0;
      }
      if (same) {
        found = (int)r.cls;
        break;
      }
    }
    if (found < 0) {
      found = (int)nc++;
      cand.push_back(Rep{std::move(g), (uint32_t)found});
    }
    class_of[i] = (uint32_t)found;
  }
  *n_classes = nc;
  return OWL_OK;
}

namespace {

/* kernel leaks: unaligned invocations, or aligned with different counts (reading R12), in alignment
   order */
void kernel_leaks(const owl_adcfg* f, const owl_adcfg* r, const Alignment& al, std::vector<owl_leak>& out) {
  const uint32_t NA = 0xFFFFFFFFu;
  const double nan = std::nan("");
  for (const OwlEdit& o : al.ops) {
    owl_leak l;
    memset(&l, 0, sizeof l);
    l.kind = OWL_LEAK_KERNEL;
    l.bb = l.ins = l.j = NA;
    l.D = l.p = nan;
    if (o.op == OWL_EDIT_DEL) {
      const uint32_t s = f->slots.order[o.i];
      l.slot_fix = s; l.slot_rnd = NA; l.kernel_id = f->slots.kid[s]; l.n = f->slots.count[s]; l.m = 0;
      out.push_back(l);
    } else if (o.op == OWL_EDIT_INS) {
      const uint32_t s = r->slots.order[o.j];
      l.slot_fix = NA; l.slot_rnd = s; l.kernel_id = r->slots.kid[s]; l.n = 0; l.m = r->slots.count[s];
      out.push_back(l);
    } else {
      const uint32_t sf = f->slots.order[o.i], sr = r->slots.order[o.j];
      const unsigned __int128 lhs = (unsigned __int128)f->slots.count[sf] * r->slots.n_runs;
      const unsigned __int128 rhs = (unsigned __int128)r->slots.count[sr] * f->slots.n_runs;
      if (lhs != rhs) {
        l.slot_fix = sf; l.slot_rnd = sr; l.kernel_id = f->slots.kid[sf];
        l.n = f->slots.count[sf]; l.m = r->slots.count[sr];
        out.push_back(l);
      }
    }
  }
}

/* CF rows, then DF rows, each by (alignment position of the fix slot, bb, ins); a DF location keeps its
   min-p row, ties -> smallest j (reading R14).  `rows` may hold several rows of one DF location (owners of
   the multi-GPU path split its visits j); CF rows are unique per (slot, bb). */
void order_ks_leaks(const Alignment& al, std::vector<owl_leak>& rows, std::vector<owl_leak>& out) {
  auto pos = [&](const owl_leak& l) { return l.slot_fix < al.pos_of_f.size() ? al.pos_of_f[l.slot_fix] : -1; };
  std::vector<owl_leak> cf, df;
  for (const owl_leak& l : rows) (l.kind == OWL_LEAK_CONTROL_FLOW ? cf : df).push_back(l);
  std::stable_sort(cf.begin(), cf.end(), [&](const owl_leak& a, const owl_leak& b) {
    return std::make_tuple(pos(a), a.bb) < std::make_tuple(pos(b), b.bb);
  });
  std::stable_sort(df.begin(), df.end(), [&](const owl_leak& a, const owl_leak& b) {
    return std::make_tuple(pos(a), a.bb, a.ins, a.p, a.j) < std::make_tuple(pos(b), b.bb, b.ins, b.p, b.j);
  });
  out.insert(out.end(), cf.begin(), cf.end());
  for (size_t i = 0; i < df.size(); ++i) /* first of each location = min p, then smallest j */
    if (i == 0 || pos(df[i]) != pos(df[i - 1]) || df[i].bb != df[i - 1].bb || df[i].ins != df[i - 1].ins)
      out.push_back(df[i]);
}

}  // namespace

OWL_API owl_status owl_leak_test(owl_ctx* ctx, const owl_adcfg* f, const owl_adcfg* r, double significance,
                                 owl_leak** leaks, size_t* n_leaks) {
  OWL_RANGE();
  if (!ctx || !f || !r || !leaks || !n_leaks) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  const uint32_t NA = 0xFFFFFFFFu;
  Alignment al = align(f, r);
  std::vector<owl_leak> out;
  kernel_leaks(f, r, al, out);
  std::vector<owl_ks_row> rows;
  std::vector<int> pos;
  owl_status s = run_ks(ctx, f, r, significance, al, rows, pos);
  if (s != OWL_OK) return s;
  auto to_leak = [&](const owl_ks_row& k, uint32_t kind) {
    owl_leak l;
    l.kind = kind; l.slot_fix = k.slot_fix; l.slot_rnd = k.slot_rnd; l.bb = k.bb;
    l.ins = kind == OWL_LEAK_DATA_FLOW ? k.ins : NA;
    l.j = kind == OWL_LEAK_DATA_FLOW ? k.j : NA;
    l.kernel_id = f->slots.kid[k.slot_fix];
    l.n = k.n; l.m = k.m; l.K_lo = k.K_lo; l.K_hi = k.K_hi; l.D = k.D; l.p = k.p;
    return l;
  };
  /* CF leaks at the node's BB; DF leak at (slot, bb, ins) if any visit j fails, representative =
     min p, ties -> smallest j (R14) */
  std::vector<owl_leak> failing;
  for (const owl_ks_row& k : rows)
    if (k.fail) failing.push_back(to_leak(k, k.kind));
  order_ks_leaks(al, failing, out);
  *leaks = host_copy(out);
  *n_leaks = out.size();
  return OWL_OK;
}

OWL_API owl_status owl_merge_leaks(owl_ctx* ctx, const owl_adcfg* f, const owl_adcfg* r, const owl_leak* parts,
                                   size_t n_parts, owl_leak** leaks, size_t* n_leaks) {
  OWL_RANGE();
  if (!ctx || !f || !r || !leaks || !n_leaks || (n_parts && !parts)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  Alignment al = align(f, r);
  std::vector<owl_leak> out, ks;
  kernel_leaks(f, r, al, out); /* replicated on every owner: recomputed here from the slot tables */
  for (size_t i = 0; i < n_parts; ++i) {
    const owl_leak& l = parts[i];
    if (l.kind == OWL_LEAK_KERNEL) continue;
    if (l.kind > OWL_LEAK_DATA_FLOW || l.slot_fix >= al.pos_of_f.size() || al.pos_of_f[l.slot_fix] < 0)
      return fail(OWL_ERR_INVALID_ARG, "leak row %zu: kind %u / fix slot %u not an aligned slot of e_fix", i, l.kind,
                  l.slot_fix);
    ks.push_back(l);
  }
  order_ks_leaks(al, ks, out);
  *leaks = host_copy(out);
  *n_leaks = out.size();
  return OWL_OK;
}

OWL_API owl_status owl_merge_diffs(owl_ctx* ctx, const owl_adcfg* a, const owl_adcfg* b, const owl_diff* parts,
                                   size_t n_parts, owl_diff** rows, size_t* n_rows) {
  OWL_RANGE();
  if (!ctx || !a || !b || !rows || !n_rows || (n_parts && !parts)) return fail(OWL_ERR_INVALID_ARG, "NULL argument");
  std::vector<owl_diff> out;
  for (size_t i = 0; i < n_parts; ++i) {
    if (parts[i].table > OWL_TABLE_SLOT) return fail(OWL_ERR_INVALID_ARG, "diff row %zu: table %u", i, parts[i].table);
    if (parts[i].table != OWL_TABLE_SLOT) out.push_back(parts[i]);
  }
  /* canonical (table, key) order: the owners' rows are disjoint (each cell lives on one owner) */
  auto key = [](const owl_diff& d) {
    return d.table == OWL_TABLE_NODE   ? std::make_tuple(d.table, d.slot, d.bb, 0u, 0u, 0u, 0u, (uint64_t)0)
           : d.table == OWL_TABLE_EDGE ? std::make_tuple(d.table, d.slot, d.prev, d.next, 0u, 0u, 0u, (uint64_t)0)
           : d.table == OWL_TABLE_TRIPLE ? std::make_tuple(d.table, d.slot, d.bb, d.prev, d.next, 0u, 0u, (uint64_t)0)
                                         : std::make_tuple(d.table, d.slot, d.bb, d.ins, d.j, 0u, 0u, d.x);
  };
  std::sort(out.begin(), out.end(), [&](const owl_diff& x, const owl_diff& y) { return key(x) < key(y); });
  /* slot rows (replicated): recomputed from the slot tables, exactly as owl_diff_adcfg writes them */
  {
    std::map<std::pair<uint32_t, uint64_t>, std::pair<uint64_t, uint64_t>> all;
    for (uint32_t sl : a->slots.order) all[{sl, a->slots.kid[sl]}].first = a->slots.count[sl];
    for (uint32_t sl : b->slots.order) all[{sl, b->slots.kid[sl]}].second = b->slots.count[sl];
    for (auto& e : all)
      if (e.second.first != e.second.second) {
        owl_diff r;
        memset(&r, 0, sizeof r);
        r.table = OWL_TABLE_SLOT;
        r.slot = e.first.first;
        r.bb = r.ins = r.j = r.prev = r.next = 0xFFFFFFFFu;
        r.x = e.first.second;
        r.count_a = e.second.first;
        r.count_b = e.second.second;
        out.push_back(r);
      }
  }
  *rows = host_copy(out);
  *n_rows = out.size();
  return OWL_OK;
}

OWL_API owl_status owl_partition_evidence(owl_ctx* ctx, const owl_adcfg* partial, int world, void** d_send,
                                          uint64_t* send_bytes) {
  OWL_RANGE();
  if (!ctx || !partial || world < 1 || !d_send || !send_bytes) return fail(OWL_ERR_INVALID_ARG, "bad argument");
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  owl_adcfg* g = const_cast<owl_adcfg*>(partial);
  if (g->send) { owl_dev_free(g->send); g->send = nullptr; }
  std::vector<uint64_t> counts(world);
  bool tables = true; /* pack straight from the hash tables; an evidence that kept only its sorted cells uses those */
  for (int t = 0; t < T_NUM; ++t) tables = tables && g->tab[t].b;
  if (tables) {
    CUDA_TRY(owl_partition_tables(g->tab, world, &g->send, counts.data(), ctx->stream), "partition");
  } else {
    owl_status s = ensure_sorted(g);
    if (s != OWL_OK) return s;
    CUDA_TRY(owl_partition_cells(g->sorted, world, &g->send, counts.data(), ctx->stream), "partition");
  }
  for (int w = 0; w < world; ++w) send_bytes[w] = counts[w] * sizeof(ExchangeCell);
  *d_send = g->send;
  return OWL_OK;
}

OWL_API owl_status owl_absorb_evidence(owl_ctx* ctx, const owl_adcfg* like, const void* d_recv, const uint64_t* recv_bytes,
                                       int world, int rank, owl_adcfg** owned) {
  OWL_RANGE();
  (void)rank;
  if (!ctx || !like || world < 1 || !owned || !recv_bytes) return fail(OWL_ERR_INVALID_ARG, "bad argument");
  CUDA_TRY(cudaSetDevice(ctx->device), "cudaSetDevice");
  uint64_t total = 0;
  for (int w = 0; w < world; ++w) {
    if (recv_bytes[w] % sizeof(ExchangeCell)) return fail(OWL_ERR_INVALID_ARG, "recv_bytes[%d] not a multiple of %zu", w, sizeof(ExchangeCell));
    total += recv_bytes[w] / sizeof(ExchangeCell);
  }
  if (total && !d_recv) return fail(OWL_ERR_INVALID_ARG, "d_recv is NULL");
  owl_adcfg* g = new owl_adcfg();
  g->ctx = ctx;
  g->cls = like->cls;
  g->slots = like->slots;
  g->max_run = like->max_run;
  g->n_records = like->n_records;
  for (int t = 0; t < T_NUM; ++t) {
    cudaError_t e = owl_table_alloc(&g->tab[t], next_pow2(2 * total + 1024), ctx->stream);
    if (e != cudaSuccess) { delete g; return cuda_fail(e, "absorb: tables"); }
  }
  cudaError_t e = cudaMemsetAsync(ctx->d_status, 0, sizeof(FoldStatus), ctx->stream);
  if (e == cudaSuccess) e = owl_absorb_cells(g->tab, (const ExchangeCell*)d_recv, total, ctx->d_status, ctx->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
  if (e != cudaSuccess) { delete g; return cuda_fail(e, "absorb"); }
  *owned = g;
  return OWL_OK;
}

/* Library statistics for measurement (not part of the analysis): fold launches, last fold duration
   (CUDA events on the context stream around the fold kernel) and records. */
OWL_API owl_status owl_get_stats(const owl_ctx* ctx, uint64_t* fold_launches, double* last_fold_ms,
                                 uint64_t* last_fold_records, double* total_fold_ms, uint64_t* total_fold_records) {
  if (!ctx) return fail(OWL_ERR_INVALID_ARG, "NULL ctx");
  if (fold_launches) *fold_launches = ctx->fold_launches;
  if (last_fold_ms) *last_fold_ms = ctx->last_fold_ms;
  if (last_fold_records) *last_fold_records = ctx->last_fold_records;
  if (total_fold_ms) *total_fold_ms = ctx->total_fold_ms;
  if (total_fold_records) *total_fold_records = ctx->total_fold_records;
  return OWL_OK;
}

OWL_API owl_status owl_reset_stats(owl_ctx* ctx) {
  if (!ctx) return fail(OWL_ERR_INVALID_ARG, "NULL ctx");
  ctx->fold_launches = 0;
  ctx->last_fold_ms = ctx->total_fold_ms = 0;
  ctx->last_fold_records = ctx->total_fold_records = 0;
  return OWL_OK;
}
