/*
 * owl_myers.cpp — A4 / A7 alignment of kernel-invocation sequences with Myers' O(ND) difference algorithm
 * (§VII.A; E. W. Myers, "An O(ND) Difference Algorithm and Its Variations", 1986), host side.
 *
 * Canonical variant (reading R11): greedy forward search over D = 0, 1, ...; on diagonal k
 * the path comes down from k+1 (an insertion of b[y]) iff k == -D or (k != D and V[k-1] < V[k+1]),
 * otherwise right from k-1 (a deletion of a[x]); then the snake of matches; the search stops at the first
 * diagonal that reaches x >= N and y >= M.  The script is recovered by walking the per-D frontiers back
 * from (N, M), then normalized so that inside every maximal run of non-matching operations the deletions
 * come before the insertions.
 */
#include <cstdint>
#include <vector>

#include "owl_myers.h"

std::vector<OwlEdit> owl_myers(const std::vector<uint64_t>& a, const std::vector<uint64_t>& b) {
  const long N = (long)a.size(), M = (long)b.size();
  /* frontier of step D lives at hist[D] (2D+1 diagonals k = -D..D at index k + D); frontier "-1" is the
     virtual start V[1] = 0 */
  std::vector<std::vector<long>> hist;
  auto get = [&](long D, long k) -> long { /* V_D[k]; for D = -1 only k = 1 exists (value 0) */
    if (D < 0) return 0;
    return hist[D][k + D];
  };
  long Dend = -1, kend = 0;
  for (long D = 0; Dend < 0; ++D) {
    hist.emplace_back(2 * D + 1, 0);
    for (long k = -D; k <= D; k += 2) {
      long x;
      const bool down = (k == -D) || (k != D && get(D - 1, k - 1) < get(D - 1, k + 1));
      if (D == 0) x = 0;
      else x = down ? get(D - 1, k + 1) : get(D - 1, k - 1) + 1;
      long y = x - k;
      while (x < N && y < M && a[x] == b[y]) { ++x; ++y; }
      hist[D][k + D] = x;
      if (x >= N && y >= M) { Dend = D; kend = k; break; }
    }
  }
  (void)kend;
  std::vector<OwlEdit> rev;
  long x = N, y = M;
  for (long D = Dend; D > 0; --D) {
    const long k = x - y;
    const bool down = (k == -D) || (k != D && get(D - 1, k - 1) < get(D - 1, k + 1));
    const long pk = down ? k + 1 : k - 1;
    const long px = get(D - 1, pk), py = px - pk;
    const long sx = down ? px : px + 1; /* the point right after the non-diagonal step */
    while (x > sx) { rev.push_back({OWL_EDIT_MATCH, (int)(x - 1), (int)(y - 1)}); --x; --y; }
    if (down) rev.push_back({OWL_EDIT_INS, -1, (int)py});
    else rev.push_back({OWL_EDIT_DEL, (int)px, -1});
    x = px;
    y = py;
  }
  while (x > 0) { rev.push_back({OWL_EDIT_MATCH, (int)(x - 1), (int)(y - 1)}); --x; --y; }
  std::vector<OwlEdit> out;
  out.reserve(rev.size());
  /* normalization while restoring forward order */
  size_t i = rev.size();
  while (i > 0) {
    if (rev[i - 1].op == OWL_EDIT_MATCH) { out.push_back(rev[i - 1]); --i; continue; }
    size_t j = i;
    while (j > 0 && rev[j - 1].op != OWL_EDIT_MATCH) --j; /* [j, i) is one non-matching stretch (reversed) */
    for (size_t q = i; q > j; --q) if (rev[q - 1].op == OWL_EDIT_DEL) out.push_back(rev[q - 1]);
    for (size_t q = i; q > j; --q) if (rev[q - 1].op == OWL_EDIT_INS) out.push_back(rev[q - 1]);
    i = j;
  }
  return out;
}
