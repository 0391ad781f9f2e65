#define KT float
#define KFN group_fn_f32
#include "k_group.inc"
