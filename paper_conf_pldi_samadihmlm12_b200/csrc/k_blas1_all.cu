#define B1OP adaptic::B1_ALL
#define B1_GROUP_FN b1_group_fn_all
#define B1_CTA_FN b1_cta_fn_all
#include "k_blas1.inc"
