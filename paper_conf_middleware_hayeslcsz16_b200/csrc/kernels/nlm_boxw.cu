// nlm_boxw.cu -- nlm_box.cu's NLM kernel with 128-column output tiles (NLMB_WIDE): every
// phase-B thread owns an output column and a 2048-wide frame is 16 tile columns (1440 tiles =
// 4.9 waves of 296 CTA slots at k = 2, instead of 1530 = 5.2).  Same arithmetic per value.
#define NLMB_WIDE 1
#include "nlm_box.cu"
