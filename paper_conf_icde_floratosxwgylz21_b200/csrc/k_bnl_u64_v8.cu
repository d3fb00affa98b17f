// k_bnl_u64_v8.cu -- block-nested-loop kernels, uint64_t keys, 8-byte payload.
#define NG_K uint64_t
#define NG_VB 8
#define NG_FAMILY_FN bnl_family_u64_v8
#include "k_bnl_family.inc"
