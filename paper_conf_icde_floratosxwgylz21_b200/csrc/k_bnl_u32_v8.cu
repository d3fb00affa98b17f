// k_bnl_u32_v8.cu -- block-nested-loop kernels, uint32_t keys, 8-byte payload.
#define NG_K uint32_t
#define NG_VB 8
#define NG_FAMILY_FN bnl_family_u32_v8
#include "k_bnl_family.inc"
