// k_bnl_u64_v4.cu -- block-nested-loop kernels, uint64_t keys, 4-byte payload.
#define NG_K uint64_t
#define NG_VB 4
#define NG_FAMILY_FN bnl_family_u64_v4
#include "k_bnl_family.inc"
