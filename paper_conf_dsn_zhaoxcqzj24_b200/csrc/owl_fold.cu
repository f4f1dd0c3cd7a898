/* owl_fold.cu — the fold kernel over warp-major segments (A1-A3; owl_fold_body.cuh holds the design and the code,
   shared with owl_fold_burst.cu, which walks channel-order segments in place through their burst index). */
#define FOLD_BURST 0
#include "owl_fold_body.cuh"
