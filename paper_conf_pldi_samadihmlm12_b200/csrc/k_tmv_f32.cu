#define KT float
#define KFN tmv_fn_f32
#include "k_tmv.inc"
