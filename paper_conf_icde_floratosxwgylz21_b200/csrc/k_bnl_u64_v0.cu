// k_bnl_u64_v0.cu -- block-nested-loop kernels, uint64_t keys, 0-byte payload.
#define NG_K uint64_t
#define NG_VB 0
#define NG_FAMILY_FN bnl_family_u64_v0
#include "k_bnl_family.inc"
