#define KT float
#define KFN tmv_mis_fn_f32
#include "k_tmv_mis.inc"
