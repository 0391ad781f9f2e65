#define KT uint32_t
#define KFN tmv_mis_fn_i32
#include "k_tmv_mis.inc"
