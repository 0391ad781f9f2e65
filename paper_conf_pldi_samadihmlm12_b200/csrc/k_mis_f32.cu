#define KT float
#define MIS_GROUP_FN mis_group_fn_f32
#define MIS_CTA_FN mis_cta_fn_f32
#define MIS_SHIFT_FN mis_shift_fn_f32
#define MIS_CTA_RB_FN mis_cta_rb_fn_f32
#define MIS_CTA_FX_FN mis_cta_fx_fn_f32
#include "k_mis.inc"
