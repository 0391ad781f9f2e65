#define B1OP adaptic::B1_NRM2
#define B1_GROUP_FN b1_group_fn_nrm2
#define B1_CTA_FN b1_cta_fn_nrm2
#include "k_blas1.inc"
