// k_bnl_u32_v0.cu -- block-nested-loop kernels, uint32_t keys, 0-byte payload.
#define NG_K uint32_t
#define NG_VB 0
#define NG_FAMILY_FN bnl_family_u32_v0
#include "k_bnl_family.inc"
