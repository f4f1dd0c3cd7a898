/* owl_fold_burst.cu — the fold kernel over channel-order segments walked in place (N2): the same walk and group-by
   as owl_fold.cu (owl_fold_body.cuh), each segment's records read through its burst index (FoldBurst). */
#define FOLD_BURST 1
#include "owl_fold_body.cuh"
