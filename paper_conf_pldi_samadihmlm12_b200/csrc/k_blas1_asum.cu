#define B1OP adaptic::B1_ASUM
#define B1_GROUP_FN b1_group_fn_asum
#define B1_CTA_FN b1_cta_fn_asum
#include "k_blas1.inc"
