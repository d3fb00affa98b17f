// k_bnl_u32_v4.cu -- block-nested-loop kernels, uint32_t keys, 4-byte payload.
#define NG_K uint32_t
#define NG_VB 4
#define NG_FAMILY_FN bnl_family_u32_v4
#include "k_bnl_family.inc"
