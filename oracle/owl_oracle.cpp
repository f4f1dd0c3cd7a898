/*
 * owl_oracle.cpp — CPU ORACLE for the Owl hot path.  TEST INFRASTRUCTURE ONLY: it may be loaded only by
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs.  The product
 * (libowl.so) never calls it, and the two share no code, header, table or helper; only the seeded
 * input generator (tracegen/) feeds both.
 *
 * A plain, slow, obviously correct implementation of what the path computes, written from the paper
 * (reference/PAPER.md, cited as P:L<n>) in the paper's order and notation:
 *   O1-O3  per-run A-DCFG: per-warp walk of the records, ordered maps            (§V.A-B)
 *   O4     evidence: runs merged in run order with Myers alignment of the kernel
 *          sequences, counts summed                                              (§VII.A)
 *   O5     diff: full outer join of two A-DCFGs                                  (§VI)
 *   O6     kernel leak test                                                      (§VII.C)
 *   O7     KS test per H_cf (node) and per H_addr (bb, ins, j)                   (Eqs. 1-8)
 *   O8     leak localization
 * Readings of ambiguous passages (R1..R20) are those of DESIGN.md §3.  fp64 arithmetic in the fixed
 * operation order of O7; compiled with -ffp-contract=off (no FMA contraction).
 *
 * Pins (tests/test_oracle_*.py): the hand-worked trace W1 (tests/golden/w1.json), conservation laws of
 * Eqs. 5-6, interleaving / lane / warp-relabel invariance, an independent pure-Python
 * per-warp walk on random tiny traces, scipy.stats.ks_2samp and exact Fraction sup for D, the KS
 * closed forms (D = 0 => p = 2; disjoint supports), Eq. 3 <=> Eq. 4, Myers against DP-LCS and script
 * validity, and the Myers examples M1-M3.
 */
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <thread>
#include <tuple>
#include <vector>

namespace {

typedef unsigned __int128 u128;
const uint32_t S = 0xFFFFFFFFu;    /* special start/end basic block (R7) */
const uint32_t NONE = 0xFFFFFFFEu; /* "no basic block entered yet" (never a valid 18-bit bb id) */
const uint32_t NA = 0xFFFFFFFFu;   /* not-applicable field */

}  // namespace

extern "C" {

/* Oracle-side record / segment / row layouts (same byte layout as the spec in DESIGN.md §5). */
typedef struct {
  uint64_t addr;
  uint32_t gwarp;
  uint32_t meta;
} orc_record;

typedef struct {
  uint32_t run, input_class, seq, n_warps;
  uint64_t kernel_id, n_records;
  const orc_record* records; /* host */
} orc_segment;

typedef struct {
  uint32_t table, slot, bb, ins, j, prev, next, _pad;
  uint64_t x, count_a, count_b;
} orc_diff_row;

typedef struct {
  uint32_t kind, slot_fix, slot_rnd, bb, ins, j;
  uint64_t kernel_id, n, m, K_lo, K_hi;
  double D, p;
} orc_leak;

typedef struct {
  uint32_t kind, slot_fix, slot_rnd, bb, ins, j;
  uint64_t n, m, K_lo, K_hi;
  double D, p;
  uint32_t fail, _pad;
} orc_ks_row;

}  // extern "C"

namespace {

typedef std::tuple<uint32_t, uint32_t> K2;                           /* node   (slot, bb)            */
typedef std::tuple<uint32_t, uint32_t, uint32_t> K3;                 /* edge   (slot, src, dst)      */
typedef std::tuple<uint32_t, uint32_t, uint32_t, uint32_t> K4;       /* triple (slot, bb, prev, next)*/
typedef std::tuple<uint32_t, uint32_t, uint32_t, uint32_t, uint64_t> K5; /* addr (slot, bb, ins, j, x)*/

/* An A-DCFG of one run, or an evidence. */
struct Adcfg {
  uint32_t input_class = 0;
  uint32_t n_runs = 0;
  std::vector<uint32_t> order;      /* ordered slot list (evidence order) */
  std::vector<uint64_t> slot_kid;   /* kernel_id by slot id */
  std::vector<uint64_t> slot_count; /* invocation count by slot id */
  std::map<K2, uint64_t> node;
  std::map<K3, uint64_t> edge;
  std::map<K4, uint64_t> triple;
  std::map<K5, uint64_t> addr;
  uint32_t max_run = 0; /* incremental builds: the last run merged */
};

struct BadRecord {
  bool any = false;
  uint32_t run = 0, seq = 0;
  uint64_t index = 0;
  std::string why;
  void note(uint32_t r, uint32_t s, uint64_t i, const char* w) {
    if (!any || std::make_tuple(r, s, i) < std::make_tuple(run, seq, index)) {
      any = true; run = r; seq = s; index = i; why = w;
    }
  }
};

/* Record fields (record format) */
inline uint32_t kind_of(const orc_record& r) { return r.meta >> 31; }
inline uint32_t lane_of(const orc_record& r) { return (r.meta >> 26) & 31u; }
inline uint32_t bb_of(const orc_record& r) { return (r.meta >> 8) & 0x3FFFFu; }
inline uint32_t ins_of(const orc_record& r) { return r.meta & 0xFFu; }
inline uint32_t mtype_of(const orc_record& r) { return (uint32_t)(r.addr >> 60); }

/* O1-O3: per-run A-DCFG.  For each segment of the run (ascending seq): bucket the records by gwarp,
   stably (only per-warp program order is meaningful, R17; warps are simultaneous), then walk
   each warp's trace T_w = (T_b1, T_b2, ...) keeping cur, prev and per-BB visit counts. */
void build_run(const std::vector<const orc_segment*>& segs, Adcfg& g, BadRecord& bad) {
  g.n_runs = 1;
  for (const orc_segment* sg : segs) {
    const uint32_t slot = sg->seq; /* per-run A-DCFG: slot = invocation index */
    /* stable bucket by gwarp, preserving stream order inside each warp (O1) */
    std::map<uint32_t, std::vector<uint64_t>> warps;
    for (uint64_t i = 0; i < sg->n_records; ++i) {
      const orc_record& r = sg->records[i];
      if (r.gwarp >= sg->n_warps) { bad.note(sg->run, sg->seq, i, "gwarp >= n_warps"); continue; }
      warps[r.gwarp].push_back(i);
    }
    for (auto& w : warps) {
      /* O2: the warp-level walk; counts are warp visits for nodes / edges / triples and
         thread accesses for addresses (R10). */
      uint32_t cur = NONE, prev = S;
      std::map<uint32_t, uint32_t> visits; /* j: per-warp visit ordinal of each BB (R8) */
      for (uint64_t i : w.second) {
        const orc_record& r = sg->records[i];
        if (kind_of(r) == 0) { /* BB_ENTRY */
          if (r.addr != 0 || ins_of(r) != 0 || lane_of(r) != 0) {
            bad.note(sg->run, sg->seq, i, "non-zero addr/lane/ins on a BB_ENTRY");
            continue;
          }
          const uint32_t b = bb_of(r);
          if (cur == NONE) {
            g.edge[K3(slot, S, b)] += 1;           /* start edge S -> first BB */
          } else {
            g.edge[K3(slot, cur, b)] += 1;         /* edge cur -> b */
            g.triple[K4(slot, cur, prev, b)] += 1; /* node cur entered from prev, left to b */
            prev = cur;
          }
          cur = b;
          visits[b] += 1;
          g.node[K2(slot, b)] += 1;
        } else { /* MEM */
          if (mtype_of(r) > 8) { bad.note(sg->run, sg->seq, i, "unknown memory type"); continue; }
          if (cur == NONE) { bad.note(sg->run, sg->seq, i, "MEM record before the warp's first BB_ENTRY"); continue; }
          if (bb_of(r) != cur) { bad.note(sg->run, sg->seq, i, "MEM record bb != the warp's current BB"); continue; }
          g.addr[K5(slot, cur, ins_of(r), visits[cur], r.addr)] += 1; /* m_j of instruction ins */
        }
      }
      if (cur != NONE) { /* warp end: last BB -> S */
        g.edge[K3(slot, cur, S)] += 1;
        g.triple[K4(slot, cur, prev, S)] += 1;
      }
    }
    if (g.slot_kid.size() <= slot) { g.slot_kid.resize(slot + 1, 0); g.slot_count.resize(slot + 1, 0); }
    g.slot_kid[slot] = sg->kernel_id;
    g.slot_count[slot] = 1;
    g.order.push_back(slot);
  }
}

/* ---- Myers' O(ND) greedy forward difference algorithm (E. Myers 1986) ----------------------
   Edit script between sequences a (length N) and b (length M): for D = 0, 1, ... and k = -D..D step 2,
   go down (insert b[y]) iff k == -D || (k != D && V[k-1] < V[k+1]), else right (delete a[x]); follow
   the snake; stop when x >= N && y >= M; backtrack over the saved V arrays.  Normalization (R11):
   inside each maximal non-matching stretch, deletions precede insertions. */
enum OpT { OP_MATCH = 0, OP_DEL = 1, OP_INS = 2 };
struct Op { int t; int i; int j; };

std::vector<Op> myers(const std::vector<uint64_t>& a, const std::vector<uint64_t>& b) {
  const int N = (int)a.size(), M = (int)b.size(), MAX = N + M, off = MAX + 1;
  std::vector<int> V(2 * MAX + 3, 0);
  std::vector<std::vector<int>> trace;
  int Dend = -1;
  for (int D = 0; D <= MAX && Dend < 0; ++D) {
    trace.push_back(V);
    for (int k = -D; k <= D; k += 2) {
      int x = (k == -D || (k != D && V[off + k - 1] < V[off + k + 1])) ? V[off + k + 1] : V[off + k - 1] + 1;
      int y = x - k;
      while (x < N && y < M && a[x] == b[y]) { ++x; ++y; }
      V[off + k] = x;
      if (x >= N && y >= M) { Dend = D; break; }
    }
  }
  std::vector<Op> rev;
  int x = N, y = M;
  for (int d = Dend; d > 0; --d) {
    const std::vector<int>& Vp = trace[d];
    const int k = x - y;
    const int pk = (k == -d || (k != d && Vp[off + k - 1] < Vp[off + k + 1])) ? k + 1 : k - 1;
    const int px = Vp[off + pk], py = px - pk;
    while (x > px && y > py) { rev.push_back({OP_MATCH, x - 1, y - 1}); --x; --y; }
    if (pk == k + 1) rev.push_back({OP_INS, -1, py});
    else rev.push_back({OP_DEL, px, -1});
    x = px; y = py;
  }
  while (x > 0 && y > 0) { rev.push_back({OP_MATCH, x - 1, y - 1}); --x; --y; }
  std::vector<Op> ops(rev.rbegin(), rev.rend());
  /* normalization: deletions before insertions inside each non-matching stretch */
  std::vector<Op> out;
  size_t i = 0;
  while (i < ops.size()) {
    if (ops[i].t == OP_MATCH) { out.push_back(ops[i]); ++i; continue; }
    size_t e = i;
    while (e < ops.size() && ops[e].t != OP_MATCH) ++e;
    for (size_t q = i; q < e; ++q) if (ops[q].t == OP_DEL) out.push_back(ops[q]);
    for (size_t q = i; q < e; ++q) if (ops[q].t == OP_INS) out.push_back(ops[q]);
    i = e;
  }
  return out;
}

/* O4: merge one run's A-DCFG into the evidence: 1) Myers-align the evidence's ordered
   slot list with the run's kernel sequence; 2) identical invocations: count += 1 and the A-DCFGs are
   summed; 3) distinct invocations are added to the evidence as new slots, at their script position. */
void merge_run(Adcfg& ev, const Adcfg& run) {
  std::vector<uint64_t> a, b;
  for (uint32_t s : ev.order) a.push_back(ev.slot_kid[s]);
  for (uint32_t s : run.order) b.push_back(run.slot_kid[s]);
  std::vector<Op> ops = myers(a, b);
  std::vector<uint32_t> map_run_slot(run.slot_kid.size(), NA);
  std::vector<uint32_t> new_order;
  for (const Op& o : ops) {
    if (o.t == OP_MATCH) {
      const uint32_t es = ev.order[o.i];
      ev.slot_count[es] += 1;
      map_run_slot[run.order[o.j]] = es;
      new_order.push_back(es);
    } else if (o.t == OP_DEL) {
      new_order.push_back(ev.order[o.i]);
    } else {
      const uint32_t ns = (uint32_t)ev.slot_kid.size();
      ev.slot_kid.push_back(run.slot_kid[run.order[o.j]]);
      ev.slot_count.push_back(1);
      map_run_slot[run.order[o.j]] = ns;
      new_order.push_back(ns);
    }
  }
  ev.order = new_order;
  for (auto& c : run.node) ev.node[K2(map_run_slot[std::get<0>(c.first)], std::get<1>(c.first))] += c.second;
  for (auto& c : run.edge)
    ev.edge[K3(map_run_slot[std::get<0>(c.first)], std::get<1>(c.first), std::get<2>(c.first))] += c.second;
  for (auto& c : run.triple)
    ev.triple[K4(map_run_slot[std::get<0>(c.first)], std::get<1>(c.first), std::get<2>(c.first),
                 std::get<3>(c.first))] += c.second;
  for (auto& c : run.addr)
    ev.addr[K5(map_run_slot[std::get<0>(c.first)], std::get<1>(c.first), std::get<2>(c.first),
               std::get<3>(c.first), std::get<4>(c.first))] += c.second;
  ev.n_runs += 1;
}

/* ---- KS two-sample test (Eqs. 1-4) -------------------------------------------------
   Samples are histogram x-values repeated by their counts (R4).  Walking the union of both sides'
   x-values in ascending order with running sums A (fix) and B (rnd), F_X(t) = A/n and F_Y(t) = B/m
   (Eq. 1), so D = sup|F_X - F_Y| (Eq. 2) = K / (n m) with K = max |A m - B n| (exact integers). */
struct KsOut { uint64_t n, m; u128 K; double D, p; bool fail; };

template <class Cells>
KsOut ks_test(const Cells& fx, const Cells& ry, double significance) {
  /* fx, ry: ascending (x, count) lists */
  KsOut o{};
  for (auto& c : fx) o.n += c.second;
  for (auto& c : ry) o.m += c.second;
  u128 A = 0, B = 0, K = 0;
  size_t i = 0, j = 0;
  while (i < fx.size() || j < ry.size()) {
    /* next distinct t of the union */
    bool take_i = j >= ry.size() || (i < fx.size() && !(ry[j].first < fx[i].first));
    bool take_j = i >= fx.size() || (j < ry.size() && !(fx[i].first < ry[j].first));
    if (take_i) { A += fx[i].second; ++i; }
    if (take_j) { B += ry[j].second; ++j; }
    const u128 am = A * (u128)o.m, bn = B * (u128)o.n;
    const u128 diff = am > bn ? am - bn : bn - am;
    if (diff > K) K = diff;
  }
  o.K = K;
  /* fp64, in exactly this operation order (R1-R3) */
  const double nd = (double)o.n, md = (double)o.m;
  o.D = (double)K / (nd * md);                 /* Eq. 2 */
  const double w = (nd * md) / (nd + md);
  const double x = (2.0 * (o.D * o.D)) * w;
  o.p = 2.0 * std::exp(-x);                    /* Eq. 4, unclamped (R3) */
  o.fail = o.p < significance;                 /* fail iff p < 1 - confidence (R1, R2) */
  return o;
}

struct Pair { int pos; uint32_t sf, sr; };

/* O6: kernel leak test — Myers over the two evidences' ordered slot lists by kernel_id. */
void kernel_alignment(const Adcfg& f, const Adcfg& r, std::vector<Op>& ops) {
  std::vector<uint64_t> a, b;
  for (uint32_t s : f.order) a.push_back(f.slot_kid[s]);
  for (uint32_t s : r.order) b.push_back(r.slot_kid[s]);
  ops = myers(a, b);
}

/* O7 over every aligned pair: CF rows (H_cf per node, Eqs. 5-8, R5, R6) then DF rows (H_addr per
   (bb, ins, j)), each only when the attribute is present on both sides (R9). */
void all_ks(const Adcfg& f, const Adcfg& r, double sig, std::vector<orc_ks_row>& rows, std::vector<int>& pos_of) {
  std::vector<Op> ops;
  kernel_alignment(f, r, ops);
  for (size_t p = 0; p < ops.size(); ++p) {
    if (ops[p].t != OP_MATCH) continue;
    const uint32_t sf = f.order[ops[p].i], sr = r.order[ops[p].j];
    /* H_cf of each node: cells (prev, next) in row-major order of A (ascending src, then dst; S last) */
    typedef std::pair<std::pair<uint32_t, uint32_t>, uint64_t> CfCell;
    std::map<uint32_t, std::vector<CfCell>> cf_f, cf_r;
    for (auto it = f.triple.lower_bound(K4(sf, 0, 0, 0)); it != f.triple.end() && std::get<0>(it->first) == sf; ++it)
      cf_f[std::get<1>(it->first)].push_back({{std::get<2>(it->first), std::get<3>(it->first)}, it->second});
    for (auto it = r.triple.lower_bound(K4(sr, 0, 0, 0)); it != r.triple.end() && std::get<0>(it->first) == sr; ++it)
      cf_r[std::get<1>(it->first)].push_back({{std::get<2>(it->first), std::get<3>(it->first)}, it->second});
    for (auto& nf : cf_f) {
      auto nr = cf_r.find(nf.first);
      if (nr == cf_r.end()) continue;
      KsOut k = ks_test(nf.second, nr->second, sig);
      orc_ks_row row{1u, sf, sr, nf.first, NA, NA, k.n, k.m, (uint64_t)k.K, (uint64_t)(k.K >> 64), k.D, k.p,
                     k.fail ? 1u : 0u, 0u};
      rows.push_back(row);
      pos_of.push_back((int)p);
    }
    /* H_addr of each (bb, ins, j): cells x ascending */
    typedef std::pair<uint64_t, uint64_t> DfCell;
    std::map<std::tuple<uint32_t, uint32_t, uint32_t>, std::vector<DfCell>> df_f, df_r;
    for (auto it = f.addr.lower_bound(K5(sf, 0, 0, 0, 0)); it != f.addr.end() && std::get<0>(it->first) == sf; ++it)
      df_f[std::make_tuple(std::get<1>(it->first), std::get<2>(it->first), std::get<3>(it->first))].push_back(
          {std::get<4>(it->first), it->second});
    for (auto it = r.addr.lower_bound(K5(sr, 0, 0, 0, 0)); it != r.addr.end() && std::get<0>(it->first) == sr; ++it)
      df_r[std::make_tuple(std::get<1>(it->first), std::get<2>(it->first), std::get<3>(it->first))].push_back(
          {std::get<4>(it->first), it->second});
    for (auto& af : df_f) {
      auto ar = df_r.find(af.first);
      if (ar == df_r.end()) continue;
      KsOut k = ks_test(af.second, ar->second, sig);
      orc_ks_row row{2u, sf, sr, std::get<0>(af.first), std::get<1>(af.first), std::get<2>(af.first), k.n, k.m,
                     (uint64_t)k.K, (uint64_t)(k.K >> 64), k.D, k.p, k.fail ? 1u : 0u, 0u};
      rows.push_back(row);
      pos_of.push_back((int)p);
    }
  }
}

thread_local std::string g_err;

}  // namespace

extern "C" {

const char* orc_last_error(void) { return g_err.c_str(); }

/* Builds the per-run A-DCFGs (O1-O3, std::thread pool over runs) and merges them in ascending run
   order into one evidence (O4).  All segments must share input_class.  Returns NULL on a malformed
   trace (message in orc_last_error(), naming the first bad (run, seq, index)). */
void* orc_build(const orc_segment* segs, size_t n_segs, int threads) {
  std::map<uint32_t, std::vector<const orc_segment*>> runs;
  for (size_t i = 0; i < n_segs; ++i) runs[segs[i].run].push_back(&segs[i]);
  std::vector<uint32_t> run_ids;
  for (auto& r : runs) {
    std::sort(r.second.begin(), r.second.end(),
              [](const orc_segment* a, const orc_segment* b) { return a->seq < b->seq; });
    run_ids.push_back(r.first);
  }
  std::vector<Adcfg> per(run_ids.size());
  std::vector<BadRecord> bads(run_ids.size());
  std::atomic<size_t> next(0);
  int nt = threads > 0 ? threads : (int)std::max(1u, std::thread::hardware_concurrency());
  if ((size_t)nt > run_ids.size()) nt = (int)std::max<size_t>(1, run_ids.size());
  auto worker = [&]() {
    for (;;) {
      size_t i = next.fetch_add(1);
      if (i >= run_ids.size()) break;
      build_run(runs[run_ids[i]], per[i], bads[i]);
    }
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < nt; ++t) pool.emplace_back(worker);
  worker();
  for (auto& t : pool) t.join();
  BadRecord bad;
  for (auto& b : bads) if (b.any) bad.note(b.run, b.seq, b.index, b.why.c_str());
  if (bad.any) {
    char buf[256];
    snprintf(buf, sizeof buf, "malformed trace: run %u seq %u record %llu: %s", bad.run, bad.seq,
             (unsigned long long)bad.index, bad.why.c_str());
    g_err = buf;
    return nullptr;
  }
  Adcfg* ev = new Adcfg();
  ev->input_class = n_segs ? segs[0].input_class : 0;
  for (size_t i = 0; i < per.size(); ++i) {
    if (i == 0) { *ev = std::move(per[0]); ev->input_class = n_segs ? segs[0].input_class : 0; continue; }
    merge_run(*ev, per[i]);
  }
  if (per.empty()) ev->n_runs = 0;
  return ev;
}

/* Incremental form of orc_build for workloads larger than host memory (the full-size parity digests): an
   evidence starts empty; each orc_evidence_add builds the per-run A-DCFGs of a batch of runs (O1-O3, thread
   pool) and merges them into the evidence in ascending run order (O4), exactly as orc_build would after the
   runs already added.  Batches must hold runs above every run added before.  Returns 0, or -1 on a malformed
   trace or an out-of-order run (message in orc_last_error()). */
void* orc_evidence_new(uint32_t input_class) {
  Adcfg* ev = new Adcfg();
  ev->input_class = input_class;
  ev->n_runs = 0;
  return ev;
}

int orc_evidence_add(void* h, const orc_segment* segs, size_t n_segs, int threads) {
  Adcfg* ev = (Adcfg*)h;
  std::map<uint32_t, std::vector<const orc_segment*>> runs;
  for (size_t i = 0; i < n_segs; ++i) runs[segs[i].run].push_back(&segs[i]);
  if (!runs.empty() && ev->n_runs > 0 && !(runs.begin()->first > ev->max_run)) {
    g_err = "orc_evidence_add: runs must be added in ascending order";
    return -1;
  }
  std::vector<uint32_t> run_ids;
  for (auto& r : runs) {
    std::sort(r.second.begin(), r.second.end(),
              [](const orc_segment* a, const orc_segment* b) { return a->seq < b->seq; });
    run_ids.push_back(r.first);
  }
  std::vector<Adcfg> per(run_ids.size());
  std::vector<BadRecord> bads(run_ids.size());
  std::atomic<size_t> next(0);
  int nt = threads > 0 ? threads : (int)std::max(1u, std::thread::hardware_concurrency());
  if ((size_t)nt > run_ids.size()) nt = (int)std::max<size_t>(1, run_ids.size());
  auto worker = [&]() {
    for (;;) {
      size_t i = next.fetch_add(1);
      if (i >= run_ids.size()) break;
      build_run(runs[run_ids[i]], per[i], bads[i]);
    }
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < nt; ++t) pool.emplace_back(worker);
  worker();
  for (auto& t : pool) t.join();
  BadRecord bad;
  for (auto& b : bads) if (b.any) bad.note(b.run, b.seq, b.index, b.why.c_str());
  if (bad.any) {
    char buf[256];
    snprintf(buf, sizeof buf, "malformed trace: run %u seq %u record %llu: %s", bad.run, bad.seq,
             (unsigned long long)bad.index, bad.why.c_str());
    g_err = buf;
    return -1;
  }
  for (size_t i = 0; i < per.size(); ++i) { /* O4 in ascending run order; the first run of all starts the evidence */
    if (ev->n_runs == 0) {
      const uint32_t cls = ev->input_class;
      *ev = std::move(per[i]);
      ev->input_class = cls;
    } else {
      merge_run(*ev, per[i]);
    }
    ev->max_run = run_ids[i];
  }
  return 0;
}

/* Bad record location of the last failed orc_build: run, seq, index (for parity of error reports). */
void orc_free(void* h) { delete (Adcfg*)h; }

/* Canonical dump. Returns the byte size; writes when buf != NULL and cap suffices. */
size_t orc_export(void* h, void* buf, size_t cap) {
  const Adcfg& g = *(const Adcfg*)h;
  std::vector<uint8_t> out;
  auto put = [&](const void* p, size_t n) { const uint8_t* c = (const uint8_t*)p; out.insert(out.end(), c, c + n); };
  auto u32 = [&](uint32_t v) { put(&v, 4); };
  auto u64 = [&](uint64_t v) { put(&v, 8); };
  put("OWLADCFG", 8);
  u32(1); u32(g.input_class); u32(g.n_runs); u32((uint32_t)g.order.size());
  u64(g.node.size()); u64(g.edge.size()); u64(g.triple.size()); u64(g.addr.size());
  for (uint32_t s : g.order) { u32(s); u32(0); u64(g.slot_kid[s]); u64(g.slot_count[s]); }
  for (auto& c : g.node) { u32(std::get<0>(c.first)); u32(std::get<1>(c.first)); u64(c.second); }
  for (auto& c : g.edge) { u32(std::get<0>(c.first)); u32(std::get<1>(c.first)); u32(std::get<2>(c.first)); u32(0); u64(c.second); }
  for (auto& c : g.triple) {
    u32(std::get<0>(c.first)); u32(std::get<1>(c.first)); u32(std::get<2>(c.first)); u32(std::get<3>(c.first)); u64(c.second);
  }
  for (auto& c : g.addr) {
    u32(std::get<0>(c.first)); u32(std::get<1>(c.first)); u32(std::get<2>(c.first)); u32(std::get<3>(c.first));
    u64(std::get<4>(c.first)); u64(c.second);
  }
  if (buf && cap >= out.size()) memcpy(buf, out.data(), out.size());
  return out.size();
}

/* O5: full outer join of two A-DCFGs on canonical keys; rows where counts differ. */
size_t orc_diff(void* ha, void* hb, orc_diff_row* out, size_t cap) {
  const Adcfg& a = *(const Adcfg*)ha;
  const Adcfg& b = *(const Adcfg*)hb;
  std::vector<orc_diff_row> rows;
  auto join = [&](const auto& ma, const auto& mb, auto fill) {
    auto ia = ma.begin(), ib = mb.begin();
    while (ia != ma.end() || ib != mb.end()) {
      if (ib == mb.end() || (ia != ma.end() && ia->first < ib->first)) { fill(ia->first, ia->second, 0); ++ia; }
      else if (ia == ma.end() || ib->first < ia->first) { fill(ib->first, 0, ib->second); ++ib; }
      else { if (ia->second != ib->second) fill(ia->first, ia->second, ib->second); ++ia; ++ib; }
    }
  };
  join(a.node, b.node, [&](const K2& k, uint64_t ca, uint64_t cb) {
    rows.push_back({0u, std::get<0>(k), std::get<1>(k), NA, NA, NA, NA, 0u, 0ull, ca, cb}); });
  join(a.edge, b.edge, [&](const K3& k, uint64_t ca, uint64_t cb) {
    rows.push_back({1u, std::get<0>(k), NA, NA, NA, std::get<1>(k), std::get<2>(k), 0u, 0ull, ca, cb}); });
  join(a.triple, b.triple, [&](const K4& k, uint64_t ca, uint64_t cb) {
    rows.push_back({2u, std::get<0>(k), std::get<1>(k), NA, NA, std::get<2>(k), std::get<3>(k), 0u, 0ull, ca, cb}); });
  join(a.addr, b.addr, [&](const K5& k, uint64_t ca, uint64_t cb) {
    rows.push_back({3u, std::get<0>(k), std::get<1>(k), std::get<2>(k), std::get<3>(k), NA, NA, 0u, std::get<4>(k), ca, cb}); });
  std::map<std::pair<uint32_t, uint64_t>, uint64_t> sa, sb; /* (slot, kernel_id) -> invocation count */
  for (uint32_t s : a.order) sa[{s, a.slot_kid[s]}] = a.slot_count[s];
  for (uint32_t s : b.order) sb[{s, b.slot_kid[s]}] = b.slot_count[s];
  join(sa, sb, [&](const std::pair<uint32_t, uint64_t>& k, uint64_t ca, uint64_t cb) {
    rows.push_back({4u, k.first, NA, NA, NA, NA, NA, 0u, k.second, ca, cb}); });
  if (out && cap >= rows.size()) std::copy(rows.begin(), rows.end(), out);
  return rows.size();
}

/* Every KS row, in (alignment position, kind, bb, ins, j) order. */
size_t orc_ks_tests(void* hf, void* hr, double sig, orc_ks_row* out, size_t cap) {
  std::vector<orc_ks_row> rows;
  std::vector<int> pos;
  all_ks(*(const Adcfg*)hf, *(const Adcfg*)hr, sig, rows, pos);
  if (out && cap >= rows.size()) std::copy(rows.begin(), rows.end(), out);
  return rows.size();
}

/* O6-O8: located leaks, sorted kernel, CF, DF, each by (alignment position, bb, ins). */
size_t orc_leak_test(void* hf, void* hr, double sig, orc_leak* out, size_t cap) {
  const Adcfg& f = *(const Adcfg*)hf;
  const Adcfg& r = *(const Adcfg*)hr;
  const double nan = std::nan("");
  std::vector<orc_leak> kern, cf, df;
  std::vector<Op> ops;
  kernel_alignment(f, r, ops);
  for (const Op& o : ops) {
    if (o.t == OP_DEL) {
      const uint32_t s = f.order[o.i];
      kern.push_back({0u, s, NA, NA, NA, NA, f.slot_kid[s], f.slot_count[s], 0ull, 0ull, 0ull, nan, nan});
    } else if (o.t == OP_INS) {
      const uint32_t s = r.order[o.j];
      kern.push_back({0u, NA, s, NA, NA, NA, r.slot_kid[s], 0ull, r.slot_count[s], 0ull, 0ull, nan, nan});
    } else {
      const uint32_t sf = f.order[o.i], sr = r.order[o.j];
      /* aligned with different invocation counts (R12: compare count_f*R_rnd with count_r*R_fix) */
      if ((u128)f.slot_count[sf] * r.n_runs != (u128)r.slot_count[sr] * f.n_runs)
        kern.push_back({0u, sf, sr, NA, NA, NA, f.slot_kid[sf], f.slot_count[sf], r.slot_count[sr], 0ull, 0ull, nan, nan});
    }
  }
  std::vector<orc_ks_row> rows;
  std::vector<int> pos;
  all_ks(f, r, sig, rows, pos);
  /* CF leak at the node's BB; DF leak at the instruction if any visit j fails,
     reported with its minimum-p visit (ties: smallest j) (R14). */
  std::map<std::tuple<int, uint32_t, uint32_t>, size_t> df_best;
  for (size_t i = 0; i < rows.size(); ++i) {
    const orc_ks_row& k = rows[i];
    if (!k.fail) continue;
    if (k.kind == 1) {
      cf.push_back({1u, k.slot_fix, k.slot_rnd, k.bb, NA, NA, f.slot_kid[k.slot_fix], k.n, k.m, k.K_lo, k.K_hi, k.D, k.p});
    } else {
      auto key = std::make_tuple(pos[i], k.bb, k.ins);
      auto it = df_best.find(key);
      if (it == df_best.end() || k.p < rows[it->second].p) df_best[key] = i; /* rows are j-ascending */
    }
  }
  for (auto& e : df_best) {
    const orc_ks_row& k = rows[e.second];
    df.push_back({2u, k.slot_fix, k.slot_rnd, k.bb, k.ins, k.j, f.slot_kid[k.slot_fix], k.n, k.m, k.K_lo, k.K_hi, k.D, k.p});
  }
  std::vector<orc_leak> all;
  all.insert(all.end(), kern.begin(), kern.end());
  all.insert(all.end(), cf.begin(), cf.end());
  all.insert(all.end(), df.begin(), df.end());
  if (out && cap >= all.size()) std::copy(all.begin(), all.end(), out);
  return all.size();
}

/* Myers edit script, exposed for the oracle's own pins (tests): ops[i] = (type, i, j). */
size_t orc_myers(const uint64_t* a, size_t na, const uint64_t* b, size_t nb, int32_t* out, size_t cap) {
  std::vector<uint64_t> va(a, a + na), vb(b, b + nb);
  std::vector<Op> ops = myers(va, vb);
  if (out && cap >= ops.size() * 3)
    for (size_t i = 0; i < ops.size(); ++i) { out[3 * i] = ops[i].t; out[3 * i + 1] = ops[i].i; out[3 * i + 2] = ops[i].j; }
  return ops.size();
}

/* One KS test on explicit histograms (for the oracle's pins): x ascending, u64 counts. */
void orc_ks_hist(const uint64_t* xf, const uint64_t* cf, size_t nf, const uint64_t* xr, const uint64_t* cr, size_t nr,
                 double sig, orc_ks_row* out) {
  std::vector<std::pair<uint64_t, uint64_t>> f, r;
  for (size_t i = 0; i < nf; ++i) f.push_back({xf[i], cf[i]});
  for (size_t i = 0; i < nr; ++i) r.push_back({xr[i], cr[i]});
  KsOut k = ks_test(f, r, sig);
  *out = orc_ks_row{2u, NA, NA, NA, NA, NA, k.n, k.m, (uint64_t)k.K, (uint64_t)(k.K >> 64), k.D, k.p, k.fail ? 1u : 0u, 0u};
}

/* Evidence slot list (evidence order): slot ids, kernel ids, counts; returns n_slots. */
size_t orc_slots(void* h, uint32_t* slots, uint64_t* kids, uint64_t* counts, size_t cap) {
  const Adcfg& g = *(const Adcfg*)h;
  if (cap >= g.order.size())
    for (size_t i = 0; i < g.order.size(); ++i) {
      if (slots) slots[i] = g.order[i];
      if (kids) kids[i] = g.slot_kid[g.order[i]];
      if (counts) counts[i] = g.slot_count[g.order[i]];
    }
  return g.order.size();
}

}  // extern "C"
