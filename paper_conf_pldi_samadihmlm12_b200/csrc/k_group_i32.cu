#define KT uint32_t
#define KFN group_fn_i32
#include "k_group.inc"
