/* owl_device.cuh — device helpers shared by libowl's kernels: key hashing, 128-bit CAS, and the global
 * A-DCFG hash-table insert (open addressing, linear probing, 32-byte cells). */
#ifndef OWL_DEVICE_CUH
#define OWL_DEVICE_CUH
#include <cuda_runtime.h>
#include <stdint.h>

#include "owl_internal.h"

namespace owl_dev {

__device__ __forceinline__ uint64_t hmix(uint64_t hi, uint64_t lo) {
  uint64_t x = lo * 0x9E3779B97F4A7C15ull + (hi ^ (hi >> 29)) * 0xC2B2AE3D27D4EB4Full;
  x ^= x >> 31;
  x *= 0xBF58476D1CE4E5B9ull;
  x ^= x >> 29;
  return x;
}

/* Global-table home cell of a key: xor of four 32-bit multiplicative hashes of the key words, top
   log2(cap) bits, rounded down to slot 0 of its bucket; probing is linear over cells from there.  One
   definition for every kernel that probes a DevTable (fold, merge, absorb), so all agree.
   cap: power of two, 2 <= cap <= 2^31. */
__device__ __forceinline__ uint32_t tab_shift(uint64_t cap) { return (uint32_t)(33 - __ffsll((long long)cap)); }
__device__ __forceinline__ uint32_t tab_index(uint64_t hi, uint64_t lo, uint32_t shift) {
  const uint32_t h = ((uint32_t)lo * 0x9E3779B1u) ^ ((uint32_t)(lo >> 32) * 0x85EBCA77u) ^
                     ((uint32_t)hi * 0xC2B2AE3Du) ^ ((uint32_t)(hi >> 32) * 0x27D4EB2Fu);
  return (h >> shift) & ~1u;
}

__device__ __forceinline__ ulonglong2 cas128_global(unsigned long long* p, unsigned long long cmp_hi,
                                                    unsigned long long cmp_lo, unsigned long long new_hi,
                                                    unsigned long long new_lo) {
  ulonglong2 o;
  asm volatile(
      "{\n\t.reg .b128 c, n, o;\n\t"
      "mov.b128 c, {%2, %3};\n\t"
      "mov.b128 n, {%4, %5};\n\t"
      "atom.global.cas.b128 o, [%6], c, n;\n\t"
      "mov.b128 {%0, %1}, o;\n\t}"
      : "=l"(o.x), "=l"(o.y)
      : "l"(cmp_hi), "l"(cmp_lo), "l"(new_hi), "l"(new_lo), "l"(p)
      : "memory");
  return o; /* o.x = word at p (hi), o.y = word at p+8 (lo) */
}

__device__ __forceinline__ ulonglong2 cas128_shared(ulonglong2* p, unsigned long long cmp_hi, unsigned long long cmp_lo,
                                                    unsigned long long new_hi, unsigned long long new_lo) {
  ulonglong2 o;
  unsigned sp = (unsigned)__cvta_generic_to_shared(p);
  asm volatile(
      "{\n\t.reg .b128 c, n, o;\n\t"
      "mov.b128 c, {%2, %3};\n\t"
      "mov.b128 n, {%4, %5};\n\t"
      "atom.shared.cas.b128 o, [%6], c, n;\n\t"
      "mov.b128 {%0, %1}, o;\n\t}"
      : "=l"(o.x), "=l"(o.y)
      : "l"(cmp_hi), "l"(cmp_lo), "l"(new_hi), "l"(new_lo), "r"(sp)
      : "memory");
  return o;
}

__device__ __forceinline__ unsigned long long* cell_key(const DevTable& t, uint64_t i) { return &t.b[i >> 1].key[i & 1][0]; }
__device__ __forceinline__ unsigned long long* cell_count(const DevTable& t, uint64_t i) { return &t.b[i >> 1].count[i & 1]; }

__device__ __forceinline__ ulonglong2 ld_key(const unsigned long long* c) {
  ulonglong2 k;
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(k.x), "=l"(k.y) : "l"(c) : "memory");
  return k;
}

/* Insert-or-add into a global table.  Returns false (and flags overflow) if no cell was found. */
static __device__ __noinline__ bool g_insert(const DevTable& t, int tbl, uint64_t hi, uint64_t lo, uint64_t c, FoldStatus* st) {
  const uint64_t mask = t.cap - 1;
  uint64_t h = tab_index(hi, lo, tab_shift(t.cap));
  for (uint64_t probe = 0; probe < t.cap; ++probe) {
    unsigned long long* key = cell_key(t, h);
    ulonglong2 k = ld_key(key);
    if (k.x == hi && k.y == lo) {
      atomicAdd(cell_count(t, h), (unsigned long long)c);
      return true;
    }
    if (k.x == OWL_EMPTY_KEY || k.x == hi) { /* empty, being claimed, or a possibly torn read: resolve */
      ulonglong2 o = cas128_global(key, OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
      if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
        unsigned long long f = atomicAdd(t.fill, 1ull);
        if (f + 1 > (t.cap >> 1) + (t.cap >> 2)) atomicOr(&st->overflow, 1u << tbl);
        atomicAdd(cell_count(t, h), (unsigned long long)c);
        return true;
      }
      if (o.x == hi && o.y == lo) {
        atomicAdd(cell_count(t, h), (unsigned long long)c);
        return true;
      }
    }
    h = (h + 1) & mask;
  }
  atomicOr(&st->overflow, 1u << tbl);
  return false;
}


}  // namespace owl_dev
#endif
