/* owl_myers.h — Myers O(ND) alignment of kernel-invocation sequences (host). */
#ifndef OWL_MYERS_H
#define OWL_MYERS_H
#include <cstdint>
#include <vector>

enum { OWL_EDIT_MATCH = 0, OWL_EDIT_DEL = 1, OWL_EDIT_INS = 2 };
struct OwlEdit {
  int op; /* OWL_EDIT_* */
  int i;  /* index in a (match / delete), -1 otherwise */
  int j;  /* index in b (match / insert), -1 otherwise */
};
/* normalized shortest edit script turning a into b (deletions before insertions in each stretch) */
std::vector<OwlEdit> owl_myers(const std::vector<uint64_t>& a, const std::vector<uint64_t>& b);
#endif
