/*
 * owl_gen_core.h — seeded, counter-based synthetic trace generator (TEST / BENCH INFRASTRUCTURE).
 *
 * This module stands in for Owl's NVBit + Pin tracers (out of scope): it emits the
 * records a tracer would send for CUDA programs shaped like the paper's workloads (Libgpucrypto AES /
 * RSA, PyTorch ops, nvJPEG decode; §VIII, Table IV).  It is the ONE module shared by the CPU oracle
 * and the CUDA path (compiled __host__ for the oracle side, __device__ for on-GPU generation); it holds
 * none of the method's arithmetic (no folding, no counting, no statistics) — only "which warp executed
 * which basic block and touched which address".
 *
 * Every record is a pure function of (seed, config, input class, run, kernel invocation, warp, lane,
 * step) via SplitMix64, so host and device produce byte-identical traces without shipping data.
 * Record layout (16 B): see DESIGN.md §5 / include/owl.h (the layout is a format spec; this module
 * defines its own struct and includes neither side's headers).
 *
 * Workload recipes:
 *   C1 toy            1 kernel, 2 blocks x 128 thr; secret key byte; branch on key bit; T-table lookups
 *   C2 AES-128        1 kernel, 256 x 256 thr; 4 pt lds, 44 round-key lds, 9 rounds x 16 Te lookups,
 *                     16 S-box lookups, 4 ct stores (212 mem / thread, 12 BB entries / warp)
 *   C3 RSA modexp     1 kernel, 16 x 256 thr; left-to-right square-and-multiply over a 256-bit secret
 *                     exponent (FIX: popcount exactly 128)
 *   C4 PyTorch-shaped embedding (token ids secret) / conv2d / softmax / conditional nonzero kernel
 *                     (launched only if the input is not all-zero: RND all-zero with probability 1/2)
 *   C5 nvJPEG-shaped  Huffman decode (8,192 thr, image-dependent symbol counts and LUT lookups) + IDCT
 *                     (128,000 thr)
 *   9  kernel-sequence model: a secret-dependent launch sequence over the C4 kernel bodies with a
 *                     repeated kernel (3-4x) and mid-sequence insertions / a trailing deletion (Myers)
 * Runs: run r is FIX or RND interleaved (r even FIX / odd RND while both classes have runs left);
 * FIX reuses one secret for all its runs, RND draws a fresh secret per run.  Non-secret
 * inputs (plaintexts, images' geometry, conv inputs) are fixed per thread across runs.
 */
#ifndef OWL_GEN_CORE_H
#define OWL_GEN_CORE_H

#include <stdint.h>

#if defined(__CUDACC__)
#define OG_HD static __host__ __device__ __forceinline__
#else
#define OG_HD static inline
#endif

typedef struct {
  uint64_t addr;
  uint32_t gwarp;
  uint32_t meta;
} og_record;

typedef struct {
  uint32_t config;   /* 1..5 (BASELINE configs), 6..8 (RQ2 sweep), 9 (kernel-sequence model) */
  uint32_t grid_div; /* every kernel's block count is divided by this (min 1 block); 1 = paper shape */
  uint32_t runs_fix;
  uint32_t runs_rnd;
  uint64_t seed;     /* master seed; DESIGN.md default 0x4F574C21 */
  uint32_t threads;  /* configs 6-8 (RQ2 trace-size sweep): the input size = thread count */
  uint32_t _pad;
} og_params;

enum { OG_FIX = 0, OG_RND = 1 };
enum { OG_T_NONE = 0, OG_T_LOCAL = 1, OG_T_GENERIC = 2, OG_T_GLOBAL = 3, OG_T_SHARED = 4, OG_T_CONST = 5,
       OG_T_G2S = 6, OG_T_SURFACE = 7, OG_T_TEXTURE = 8 };

/* stream tags of the counter-based generator */
enum { OG_TAG_FIX = 1, OG_TAG_RND, OG_TAG_PT, OG_TAG_NOISE, OG_TAG_STATE, OG_TAG_EXP, OG_TAG_TOK, OG_TAG_ZERO,
       OG_TAG_NS, OG_TAG_CODE, OG_TAG_KID, OG_TAG_PERM, OG_TAG_SEQ };

OG_HD uint64_t og_mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
OG_HD uint64_t og_h2(uint64_t a, uint64_t b) { return og_mix(og_mix(a) ^ b); }
OG_HD uint64_t og_h3(uint64_t a, uint64_t b, uint64_t c) { return og_mix(og_h2(a, b) ^ c); }
OG_HD uint64_t og_h4(uint64_t a, uint64_t b, uint64_t c, uint64_t d) { return og_mix(og_h3(a, b, c) ^ d); }

OG_HD uint64_t og_addr(uint32_t type, uint32_t alloc, uint64_t off) {
  return ((uint64_t)type << 60) | ((uint64_t)(alloc & 0xFFFFu) << 44) | (off & ((1ull << 44) - 1));
}

/* ---- runs and classes ---------------------------------------------------------------------------- */
OG_HD uint32_t og_n_runs(const og_params* p) { return p->runs_fix + p->runs_rnd; }
OG_HD uint32_t og_run_class(const og_params* p, uint32_t r) {
  uint32_t mn = p->runs_fix < p->runs_rnd ? p->runs_fix : p->runs_rnd;
  if (r < 2 * mn) return r & 1u;
  return p->runs_fix > p->runs_rnd ? OG_FIX : OG_RND;
}
/* secret of a run: one for all FIX runs, a fresh one per RND run */
OG_HD uint64_t og_run_secret(const og_params* p, uint32_t r) {
  if (og_run_class(p, r) == OG_FIX) return og_h3(p->seed, OG_TAG_FIX, p->config);
  return og_h4(p->seed, OG_TAG_RND, p->config, r);
}
OG_HD uint32_t og_blocks(const og_params* p, uint32_t dflt) {
  uint32_t d = p->grid_div ? p->grid_div : 1u;
  uint32_t b = dflt / d;
  return b ? b : 1u;
}

/* ---- kernel sequence of a run ------------------------------------------------------------------- */
enum { OG_K_TOY = 0, OG_K_AES, OG_K_RSA, OG_K_EMBED, OG_K_CONV, OG_K_SOFTMAX, OG_K_NONZERO, OG_K_HUFF, OG_K_IDCT,
       OG_K_SBOX, OG_K_PIXEL, OG_K_REPR };

OG_HD int og_c4_allzero(const og_params* p, uint32_t r) {
  return p->config == 4 && og_run_class(p, r) == OG_RND && (og_h2(og_run_secret(p, r), OG_TAG_ZERO) & 1u);
}
/* config 9 (kernel-sequence model): the host code of a small model launches a secret-dependent kernel
   sequence E L [G] L [G] L [L] [N] — the layer kernel L repeats 3-4 times, the gate kernel G is inserted
   mid-sequence 0-2 times, the final N is skipped on one secret bit — so the Myers alignment of runs
    sees repeated kernel ids and mid-sequence insertions / deletions.  Returns the length. */
OG_HD uint32_t og_c9_seq(const og_params* p, uint32_t r, uint32_t* ks) {
  const uint64_t b = og_h2(og_run_secret(p, r), OG_TAG_SEQ);
  uint32_t n = 0;
  ks[n++] = OG_K_EMBED;
  ks[n++] = OG_K_SOFTMAX;
  if (b & 1u) ks[n++] = OG_K_NONZERO;
  ks[n++] = OG_K_SOFTMAX;
  if (b & 2u) ks[n++] = OG_K_NONZERO;
  ks[n++] = OG_K_SOFTMAX;
  if (b & 4u) ks[n++] = OG_K_SOFTMAX;
  if (!(b & 8u)) ks[n++] = OG_K_CONV;
  return n;
}
OG_HD uint32_t og_n_seq(const og_params* p, uint32_t r) {
  uint32_t ks[8];
  switch (p->config) {
    case 4: return og_c4_allzero(p, r) ? 3u : 4u;
    case 5: return 2u;
    case 9: return og_c9_seq(p, r, ks);
    default: return 1u;
  }
}
OG_HD uint32_t og_seq_kernel(const og_params* p, uint32_t r, uint32_t seq) {
  uint32_t ks[8];
  switch (p->config) {
    case 9: return og_c9_seq(p, r, ks) > seq ? ks[seq] : OG_K_CONV;
    case 1: return OG_K_TOY;
    case 2: return OG_K_AES;
    case 3: return OG_K_RSA;
    case 4: return seq == 0 ? OG_K_EMBED : seq == 1 ? OG_K_CONV : seq == 2 ? OG_K_SOFTMAX : OG_K_NONZERO;
    case 6: return OG_K_SBOX;
    case 7: return OG_K_PIXEL;
    case 8: return OG_K_REPR;
    default: return seq == 0 ? OG_K_HUFF : OG_K_IDCT;
  }
}
/* call-stack hash of the launch site: fixed per (config, kernel) */
OG_HD uint64_t og_kernel_id(const og_params* p, uint32_t k) { return og_h3(0x0DC0FFEEull, OG_TAG_KID, p->config * 16u + k); }
OG_HD uint32_t og_kernel_wpb(uint32_t k) { return k == OG_K_TOY ? 4u : 8u; }
OG_HD uint32_t og_kernel_blocks(const og_params* p, uint32_t k) {
  if (p->config == 9) return og_blocks(p, 16); /* 128 warps per kernel */
  switch (k) {
    case OG_K_TOY: return og_blocks(p, 2);
    case OG_K_AES: return og_blocks(p, 256);
    case OG_K_RSA: return og_blocks(p, 16);
    case OG_K_EMBED: return og_blocks(p, 256);
    case OG_K_CONV: return og_blocks(p, 1024);
    case OG_K_SOFTMAX: return og_blocks(p, 256);
    case OG_K_NONZERO: return og_blocks(p, 256);
    case OG_K_HUFF: return og_blocks(p, 32);
    case OG_K_SBOX:
    case OG_K_PIXEL: return p->threads ? (p->threads + 255u) / 256u : 1u;
    case OG_K_REPR: return 1u;
    default: return og_blocks(p, 500); /* IDCT: 500 x 256 = 128,000 threads */
  }
}
OG_HD uint32_t og_seq_n_warps(const og_params* p, uint32_t r, uint32_t seq) {
  uint32_t k = og_seq_kernel(p, r, seq);
  return og_kernel_blocks(p, k) * og_kernel_wpb(k);
}

/* ---- emitter ------------------------------------------------------------------------------------ */
typedef struct {
  og_record* out; /* NULL: count only */
  uint64_t n;
  uint32_t gwarp;
} og_em;

OG_HD void og_bb(og_em* e, uint32_t bb) {
  if (e->out) {
    og_record rec;
    rec.addr = 0;
    rec.gwarp = e->gwarp;
    rec.meta = (bb & 0x3FFFFu) << 8;
    e->out[e->n] = rec;
  }
  e->n++;
}
OG_HD void og_mem(og_em* e, uint32_t lane, uint32_t bb, uint32_t ins, uint64_t addr) {
  if (e->out) {
    og_record rec;
    rec.addr = addr;
    rec.gwarp = e->gwarp;
    rec.meta = 0x80000000u | ((lane & 31u) << 26) | ((bb & 0x3FFFFu) << 8) | (ins & 0xFFu);
    e->out[e->n] = rec;
  }
  e->n++;
}

/* ---- C1: toy kernel (one secret-dependent branch + T-table lookups) ------------------------------- */
OG_HD uint32_t og_c1_key(const og_params* p, uint32_t r) {
  uint32_t k = (uint32_t)(og_run_secret(p, r) & 0xFFu);
  if (og_run_class(p, r) == OG_FIX) k |= 1u; /* the fixed key takes the T-table branch B1 */
  return k;
}
OG_HD uint32_t og_c1_pt(const og_params* p, uint32_t tid, uint32_t i) {
  return (uint32_t)(og_h4(p->seed, OG_TAG_PT, tid, i) & 0xFFu);
}
OG_HD void og_warp_c1(const og_params* p, uint32_t r, og_em* e) {
  const uint32_t key = og_c1_key(p, r);
  const uint32_t w = e->gwarp;
  uint32_t l, i;
  og_bb(e, 0);
  for (l = 0; l < 32; ++l) og_mem(e, l, 0, 0, og_addr(OG_T_CONST, 1, 0));
  for (l = 0; l < 32; ++l) og_mem(e, l, 0, 1, og_addr(OG_T_GLOBAL, 2, 4ull * (w * 32 + l)));
  if (key & 1u) {
    og_bb(e, 1);
    for (i = 0; i < 8; ++i)
      for (l = 0; l < 32; ++l) og_mem(e, l, 1, i, og_addr(OG_T_SHARED, 0, 4ull * (og_c1_pt(p, w * 32 + l, i) ^ key)));
  } else {
    og_bb(e, 2);
    for (i = 0; i < 8; ++i)
      for (l = 0; l < 32; ++l) og_mem(e, l, 2, i, og_addr(OG_T_GLOBAL, 3, 4ull * (8ull * (w * 32 + l) + i)));
  }
  og_bb(e, 3);
  for (i = 0; i < 8; ++i)
    for (l = 0; l < 32; ++l) {
      uint32_t b = (uint32_t)(og_mix(((uint64_t)(og_c1_pt(p, w * 32 + l, i) ^ key) << 8) | i) & 0xFFu);
      og_mem(e, l, 3, i, og_addr(OG_T_SHARED, 0, 1024ull + 4ull * b));
    }
  for (l = 0; l < 32; ++l)
    og_mem(e, l, 3, 8, og_addr(OG_T_GLOBAL, 4, 4ull * (og_h4(p->seed, OG_TAG_NOISE, r, w * 32 + l) & 63u)));
  for (l = 0; l < 32; ++l) og_mem(e, l, 3, 9, og_addr(OG_T_GLOBAL, 5, 4ull * (w * 32 + l)));
}

/* ---- C2: AES-128 T-table encryption (Libgpucrypto-shaped) ------------------------------------------ */
OG_HD uint32_t og_c2_byte(uint64_t k0, uint64_t k1, uint64_t ptlo, uint64_t pthi, uint32_t round, uint32_t i) {
  uint64_t h = og_h3(k0 ^ ptlo, k1 ^ pthi, (uint64_t)round * 2u + (i >> 3));
  return (uint32_t)((h >> (8u * (i & 7u))) & 0xFFu);
}
OG_HD void og_warp_c2(const og_params* p, uint32_t r, og_em* e) {
  const uint64_t s = og_run_secret(p, r);
  const uint64_t k0 = og_h2(s, 0), k1 = og_h2(s, 1); /* 128-bit key shared by all threads */
  const uint32_t w = e->gwarp;
  uint64_t ptlo[32], pthi[32];
  uint32_t l, i, rd;
  for (l = 0; l < 32; ++l) {
    ptlo[l] = og_h3(p->seed, OG_TAG_PT, 2ull * (w * 32 + l));
    pthi[l] = og_h3(p->seed, OG_TAG_PT, 2ull * (w * 32 + l) + 1);
  }
  og_bb(e, 0);
  for (i = 0; i < 4; ++i)
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, i, og_addr(OG_T_GLOBAL, 1, 16ull * (w * 32 + l) + 4 * i));
  og_bb(e, 1);
  for (i = 0; i < 44; ++i)
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, i, og_addr(OG_T_SHARED, 2, 4ull * i));
  for (rd = 1; rd <= 9; ++rd) {
    og_bb(e, 2);
    for (i = 0; i < 16; ++i)
      for (l = 0; l < 32; ++l)
        og_mem(e, l, 2, i,
               og_addr(OG_T_SHARED, 3, 1024ull * (i & 3u) + 4ull * og_c2_byte(k0, k1, ptlo[l], pthi[l], rd, i)));
  }
  og_bb(e, 3);
  for (i = 0; i < 16; ++i)
    for (l = 0; l < 32; ++l)
      og_mem(e, l, 3, i, og_addr(OG_T_SHARED, 4, 4ull * og_c2_byte(k0, k1, ptlo[l], pthi[l], 10, i)));
  for (i = 0; i < 4; ++i)
    for (l = 0; l < 32; ++l) og_mem(e, l, 3, 16 + i, og_addr(OG_T_GLOBAL, 5, 16ull * (w * 32 + l) + 4 * i));
}

/* ---- C3: RSA modular exponentiation, left-to-right square-and-multiply ------------------------------ */
OG_HD void og_c3_exponent(const og_params* p, uint32_t r, uint64_t e4[4]) {
  uint64_t s = og_run_secret(p, r);
  uint32_t i;
  if (og_run_class(p, r) == OG_FIX) {
    /* fixed exponent with popcount exactly 128: first 128 positions of a seeded Fisher-Yates shuffle */
    uint8_t pos[256];
    for (i = 0; i < 256; ++i) pos[i] = (uint8_t)i;
    for (i = 255; i > 0; --i) {
      uint32_t j = (uint32_t)(og_h3(s, OG_TAG_PERM, i) % (i + 1u));
      uint8_t t = pos[i];
      pos[i] = pos[j];
      pos[j] = t;
    }
    e4[0] = e4[1] = e4[2] = e4[3] = 0;
    for (i = 0; i < 128; ++i) e4[pos[i] >> 6] |= 1ull << (pos[i] & 63u);
  } else {
    for (i = 0; i < 4; ++i) e4[i] = og_h3(s, OG_TAG_EXP, i);
  }
}
OG_HD void og_warp_c3(const og_params* p, uint32_t r, og_em* e) {
  uint64_t ex[4];
  const uint32_t w = e->gwarp;
  uint32_t l, i, q;
  int bit;
  og_c3_exponent(p, r, ex);
  og_bb(e, 0);
  for (q = 0; q < 4; ++q)
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, q, og_addr(OG_T_GLOBAL, 1, 16ull * (w * 32 + l) + 4 * q));
  for (bit = 255; bit >= 0; --bit) {
    og_bb(e, 1);
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, 0, og_addr(OG_T_CONST, 2, 4ull * ((uint32_t)bit >> 5)));
    og_bb(e, 2);
    for (i = 0; i < 8; ++i)
      for (l = 0; l < 32; ++l) {
        uint32_t tib = (w * 32 + l) & 255u;
        og_mem(e, l, 2, i, og_addr(OG_T_SHARED, 3, 4ull * (4u * tib + (i & 3u))));
      }
    if ((ex[bit >> 6] >> (bit & 63)) & 1u) {
      og_bb(e, 3);
      for (i = 0; i < 8; ++i)
        for (l = 0; l < 32; ++l) {
          uint32_t tib = (w * 32 + l) & 255u;
          og_mem(e, l, 3, i, og_addr(OG_T_SHARED, 3, 4096ull + 4ull * (4u * tib + (i & 3u))));
        }
    }
  }
  og_bb(e, 4);
  for (q = 0; q < 4; ++q)
    for (l = 0; l < 32; ++l) og_mem(e, l, 4, q, og_addr(OG_T_GLOBAL, 4, 16ull * (w * 32 + l) + 4 * q));
}

/* ---- C4: PyTorch-shaped ops ------------------------------------------------------------------------ */
OG_HD uint32_t og_c4_token(const og_params* p, uint32_t r, uint32_t tid) {
  if (og_c4_allzero(p, r)) return 0; /* pad */
  return (uint32_t)(og_h3(og_run_secret(p, r), OG_TAG_TOK, tid) % 50257u);
}
OG_HD void og_warp_c4(const og_params* p, uint32_t r, uint32_t k, og_em* e) {
  const uint32_t w = e->gwarp;
  uint32_t l, i, c, v;
  if (k == OG_K_EMBED) {
    uint32_t tok[32];
    int any_tok = 0, any_pad = 0;
    for (l = 0; l < 32; ++l) {
      tok[l] = og_c4_token(p, r, w * 32 + l);
      if (tok[l]) any_tok = 1; else any_pad = 1;
    }
    og_bb(e, 0);
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, 0, og_addr(OG_T_GLOBAL, 1, 4ull * (w * 32 + l)));
    if (any_tok) { /* row lookup, predicated on token != pad */
      og_bb(e, 1);
      for (i = 0; i < 16; ++i)
        for (l = 0; l < 32; ++l)
          if (tok[l]) og_mem(e, l, 1, i, og_addr(OG_T_GLOBAL, 2, 256ull * tok[l] + 16ull * i));
    }
    if (any_pad) og_bb(e, 2);
    og_bb(e, 3);
    for (i = 0; i < 16; ++i)
      for (l = 0; l < 32; ++l) og_mem(e, l, 3, i, og_addr(OG_T_GLOBAL, 3, 64ull * (w * 32 + l) + 4 * i));
  } else if (k == OG_K_CONV) {
    og_bb(e, 0);
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, 0, og_addr(OG_T_GLOBAL, 4, 4ull * (w * 32 + l)));
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, 1, og_addr(OG_T_SHARED, 5, 4ull * ((w * 32 + l) & 255u)));
    for (c = 0; c < 16; ++c) {
      og_bb(e, 1);
      for (i = 0; i < 9; ++i)
        for (l = 0; l < 32; ++l) {
          uint32_t tib = (w * 32 + l) & 255u;
          og_mem(e, l, 1, i, og_addr(OG_T_SHARED, 5, 4ull * ((tib + (i / 3u) * 16u + (i % 3u)) & 255u)));
        }
      for (i = 0; i < 9; ++i)
        for (l = 0; l < 32; ++l) og_mem(e, l, 1, 9 + i, og_addr(OG_T_CONST, 6, 4ull * (c * 9u + i)));
    }
    og_bb(e, 2);
    for (l = 0; l < 32; ++l) og_mem(e, l, 2, 0, og_addr(OG_T_GLOBAL, 7, 4ull * (w * 32 + l)));
  } else if (k == OG_K_SOFTMAX) {
    og_bb(e, 0);
    for (i = 0; i < 32; ++i)
      for (l = 0; l < 32; ++l) og_mem(e, l, 0, i, og_addr(OG_T_GLOBAL, 8, 128ull * (w * 32 + l) + 4 * i));
    for (v = 0; v < 5; ++v) {
      og_bb(e, 1);
      for (l = 0; l < 32; ++l) {
        uint32_t tib = (w * 32 + l) & 255u;
        og_mem(e, l, 1, 0, og_addr(OG_T_SHARED, 9, 4ull * (tib ^ (1u << v))));
      }
      for (l = 0; l < 32; ++l) og_mem(e, l, 1, 1, og_addr(OG_T_SHARED, 9, 4ull * ((w * 32 + l) & 255u)));
    }
    og_bb(e, 2);
    for (i = 0; i < 32; ++i)
      for (l = 0; l < 32; ++l) og_mem(e, l, 2, i, og_addr(OG_T_GLOBAL, 10, 128ull * (w * 32 + l) + 4 * i));
  } else { /* nonzero: launched only when the input is not all-zero (kernel leak) */
    og_bb(e, 0);
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, 0, og_addr(OG_T_GLOBAL, 1, 4ull * (w * 32 + l)));
    og_bb(e, 1);
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, 0, og_addr(OG_T_GLOBAL, 11, 0));
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, 1, og_addr(OG_T_GLOBAL, 12, 4ull * (w * 32 + l)));
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, 2, og_addr(OG_T_GLOBAL, 13, 4ull * (w * 32 + l)));
  }
}

/* ---- C5: nvJPEG-shaped decode (Huffman + IDCT) -------------------------------------------------------- */
OG_HD void og_warp_c5(const og_params* p, uint32_t r, uint32_t k, og_em* e) {
  const uint64_t img = og_run_secret(p, r);
  const uint32_t w = e->gwarp;
  uint32_t l, c, s;
  if (k == OG_K_HUFF) {
    uint32_t ns[32], mx = 0;
    for (l = 0; l < 32; ++l) {
      ns[l] = 48u + (uint32_t)(og_h3(img, OG_TAG_NS, w * 32 + l) & 31u); /* 48..79 symbols */
      if (ns[l] > mx) mx = ns[l];
    }
    og_bb(e, 0);
    for (l = 0; l < 32; ++l) og_mem(e, l, 0, 0, og_addr(OG_T_GLOBAL, 1, 4ull * (w * 32 + l)));
    for (s = 0; s < mx; ++s) {
      uint32_t code[32];
      int any_long = 0;
      og_bb(e, 1);
      for (l = 0; l < 32; ++l) {
        code[l] = (uint32_t)(og_h4(img, OG_TAG_CODE, w * 32 + l, s) & 0x1FFu);
        if (s < ns[l] && code[l] >= 448u) any_long = 1;
      }
      for (l = 0; l < 32; ++l)
        if (s < ns[l]) og_mem(e, l, 1, 0, og_addr(OG_T_GLOBAL, 2, 4ull * (128ull * (w * 32 + l) + s)));
      for (l = 0; l < 32; ++l)
        if (s < ns[l]) og_mem(e, l, 1, 1, og_addr(OG_T_SHARED, 3, 4ull * code[l]));
      if (any_long) {
        og_bb(e, 2);
        for (l = 0; l < 32; ++l)
          if (s < ns[l] && code[l] >= 448u) og_mem(e, l, 2, 0, og_addr(OG_T_SHARED, 3, 2048ull + 8ull * (code[l] & 63u)));
        for (l = 0; l < 32; ++l)
          if (s < ns[l] && code[l] >= 448u) og_mem(e, l, 2, 1, og_addr(OG_T_SHARED, 3, 2052ull + 8ull * (code[l] & 63u)));
      }
      og_bb(e, 3);
      for (l = 0; l < 32; ++l)
        if (s < ns[l]) og_mem(e, l, 3, 0, og_addr(OG_T_GLOBAL, 4, 4ull * (128ull * (w * 32 + l) + s)));
    }
    og_bb(e, 4);
    for (l = 0; l < 32; ++l) og_mem(e, l, 4, 0, og_addr(OG_T_GLOBAL, 5, 4ull * (w * 32 + l)));
  } else { /* IDCT: 64 coefficient loads shared within an 8x8 block, 8 qtable loads, one pixel store */
    og_bb(e, 0);
    for (c = 0; c < 64; ++c)
      for (l = 0; l < 32; ++l) og_mem(e, l, 0, c, og_addr(OG_T_GLOBAL, 4, 256ull * ((w * 32 + l) / 64u) + 4ull * c));
    for (c = 0; c < 8; ++c)
      for (l = 0; l < 32; ++l) og_mem(e, l, 0, 64 + c, og_addr(OG_T_CONST, 6, 4ull * c));
    og_bb(e, 1);
    for (l = 0; l < 32; ++l) og_mem(e, l, 1, 0, og_addr(OG_T_GLOBAL, 7, 4ull * (w * 32 + l)));
  }
}

/* ---- configs 6-8: the RQ2 trace-size workloads (Fig. 5), input size = p->threads ---------
   6 (pattern 2, "volatile threads with limited memory accesses"): the paper's dummy program, random
     lookups into a 256-entry S-box (16 per thread, byte = f(secret, thread, i)); distinct addresses
     saturate at 16 x 256 while records grow with the threads;
   7 (pattern 3, "volatile threads with unlimited memory access", nvJPEG-like): every thread loads four
     words of its own pixel and stores one; distinct addresses grow with the threads;
   8 (pattern 1, "fixed threads", Tensor.__repr__): one block of 256 threads reads a fixed set of
     elements whatever the input size.
   Threads beyond p->threads (the last block's tail) are inactive: they emit nothing. */
OG_HD void og_warp_rq2(const og_params* p, uint32_t r, uint32_t k, og_em* e) {
  const uint32_t w = e->gwarp;
  const uint32_t T = k == OG_K_REPR ? 256u : p->threads;
  uint32_t l, i;
  if (w * 32u >= T) return;
  const uint32_t act = T - w * 32u < 32u ? T - w * 32u : 32u; /* active lanes 0..act-1 */
  if (k == OG_K_SBOX) {
    const uint64_t sec = og_run_secret(p, r);
    og_bb(e, 0);
    for (i = 0; i < 16; ++i)
      for (l = 0; l < act; ++l)
        og_mem(e, l, 0, i, og_addr(OG_T_SHARED, 1, 4ull * (og_h3(sec, w * 32 + l, i) & 0xFFu)));
  } else if (k == OG_K_PIXEL) {
    og_bb(e, 0);
    for (i = 0; i < 4; ++i)
      for (l = 0; l < act; ++l) og_mem(e, l, 0, i, og_addr(OG_T_GLOBAL, 2, 16ull * (w * 32 + l) + 4 * i));
    for (l = 0; l < act; ++l) og_mem(e, l, 0, 4, og_addr(OG_T_GLOBAL, 3, 4ull * (w * 32 + l)));
  } else {
    og_bb(e, 0);
    for (i = 0; i < 8; ++i)
      for (l = 0; l < act; ++l) og_mem(e, l, 0, i, og_addr(OG_T_GLOBAL, 4, 4ull * (((w * 32 + l) * 8 + i) & 63u)));
  }
}

/* Records of traced warp `gwarp` of invocation `seq` of run `r`, in program order; returns the count.
   out == NULL counts only. */
OG_HD uint64_t og_warp(const og_params* p, uint32_t r, uint32_t seq, uint32_t gwarp, og_record* out) {
  og_em e;
  uint32_t k = og_seq_kernel(p, r, seq);
  e.out = out;
  e.n = 0;
  e.gwarp = gwarp;
  switch (p->config) {
    case 1: og_warp_c1(p, r, &e); break;
    case 2: og_warp_c2(p, r, &e); break;
    case 3: og_warp_c3(p, r, &e); break;
    case 4: case 9: og_warp_c4(p, r, k, &e); break;
    case 6: case 7: case 8: og_warp_rq2(p, r, k, &e); break;
    default: og_warp_c5(p, r, k, &e); break;
  }
  return e.n;
}

#endif /* OWL_GEN_CORE_H */
