#define KT uint32_t
#define KFN tmv_fn_i32
#include "k_tmv.inc"
