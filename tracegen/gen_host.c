/* gen_host.c — host build of the synthetic trace generator (libowlgen.so).  TEST / BENCH
 * INFRASTRUCTURE: produces warp-major records for the CPU oracle and for host-buffer (e2e) runs.
 * See owl_gen_core.h for the recipe. */
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#include "owl_gen_core.h"

#define OG_API __attribute__((visibility("default")))

OG_API uint32_t ogh_n_runs(const og_params* p) { return og_n_runs(p); }
OG_API uint32_t ogh_run_class(const og_params* p, uint32_t r) { return og_run_class(p, r); }
OG_API uint32_t ogh_n_seq(const og_params* p, uint32_t r) { return og_n_seq(p, r); }
OG_API void ogh_seq_meta(const og_params* p, uint32_t r, uint32_t seq, uint64_t* kernel_id, uint32_t* n_warps,
                         uint32_t* cls) {
  uint32_t k = og_seq_kernel(p, r, seq);
  if (kernel_id) *kernel_id = og_kernel_id(p, k);
  if (n_warps) *n_warps = og_seq_n_warps(p, r, seq);
  if (cls) *cls = og_run_class(p, r);
}

typedef struct {
  const og_params* p;
  uint32_t r, seq, w0, w1;
  uint64_t* counts;     /* per warp */
  const uint64_t* offs; /* per warp (generate pass) */
  og_record* out;
} og_job;

static void* og_job_run(void* arg) {
  og_job* j = (og_job*)arg;
  uint32_t w;
  for (w = j->w0; w < j->w1; ++w) {
    if (j->out)
      og_warp(j->p, j->r, j->seq, w, j->out + j->offs[w]);
    else
      j->counts[w] = og_warp(j->p, j->r, j->seq, w, NULL);
  }
  return NULL;
}

static void og_parallel(const og_params* p, uint32_t r, uint32_t seq, uint32_t nw, uint64_t* counts,
                        const uint64_t* offs, og_record* out, int threads) {
  pthread_t th[256];
  og_job jobs[256];
  int t, nt = threads < 1 ? 1 : (threads > 256 ? 256 : threads);
  if ((uint32_t)nt > nw) nt = nw ? (int)nw : 1;
  for (t = 0; t < nt; ++t) {
    jobs[t].p = p; jobs[t].r = r; jobs[t].seq = seq;
    jobs[t].w0 = (uint32_t)((uint64_t)nw * t / nt);
    jobs[t].w1 = (uint32_t)((uint64_t)nw * (t + 1) / nt);
    jobs[t].counts = counts; jobs[t].offs = offs; jobs[t].out = out;
  }
  if (nt == 1) { og_job_run(&jobs[0]); return; }
  for (t = 0; t < nt; ++t) pthread_create(&th[t], NULL, og_job_run, &jobs[t]);
  for (t = 0; t < nt; ++t) pthread_join(th[t], NULL);
}

/* Per-warp record counts (warp_counts may be NULL); returns the segment's record count. */
OG_API uint64_t ogh_seq_count(const og_params* p, uint32_t r, uint32_t seq, uint64_t* warp_counts, int threads) {
  uint32_t nw = og_seq_n_warps(p, r, seq), w;
  uint64_t* c = warp_counts ? warp_counts : (uint64_t*)malloc(sizeof(uint64_t) * nw);
  uint64_t tot = 0;
  og_parallel(p, r, seq, nw, c, NULL, NULL, threads);
  for (w = 0; w < nw; ++w) tot += c[w];
  if (!warp_counts) free(c);
  return tot;
}

/* Writes the segment's records warp-major (warps ascending, each in program order) to out. */
OG_API uint64_t ogh_seq_generate(const og_params* p, uint32_t r, uint32_t seq, og_record* out, int threads) {
  uint32_t nw = og_seq_n_warps(p, r, seq), w;
  uint64_t* c = (uint64_t*)malloc(sizeof(uint64_t) * nw);
  uint64_t* o = (uint64_t*)malloc(sizeof(uint64_t) * nw);
  uint64_t tot = 0;
  og_parallel(p, r, seq, nw, c, NULL, NULL, threads);
  for (w = 0; w < nw; ++w) { o[w] = tot; tot += c[w]; }
  og_parallel(p, r, seq, nw, NULL, o, out, threads);
  free(c);
  free(o);
  return tot;
}
