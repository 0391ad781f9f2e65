#define B1OP adaptic::B1_IAMIN
#define B1_GROUP_FN b1_group_fn_iamin
#define B1_CTA_FN b1_cta_fn_iamin
#include "k_blas1.inc"
