#define B1OP adaptic::B1_IAMAX
#define B1_GROUP_FN b1_group_fn_iamax
#define B1_CTA_FN b1_cta_fn_iamax
#include "k_blas1.inc"
