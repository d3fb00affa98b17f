// k_bnl.cu -- dispatch of the a7 block-nested-loop kernel families.
#include "k_bnl.cuh"

namespace ng {

// rb_done: one word per R block of the smallest block size (B_THREADS tuples)
size_t bnl_scratch_bytes(long long n_rp_max) { return 256 + (size_t)((n_rp_max + B_THREADS - 1) / B_THREADS + 1) * 4; }

cudaError_t launch_bnl(int kb, int vb, int op, int agg, long long n_rp_max, const long long *d_nrp, const void *rkeys,
                       long long ns_max, const long long *d_nsp, const void *skeys, const void *svals,
                       const unsigned *extreme, long long *acc, long long *cnt, void *scratch, int num_sms,
                       int shape, cudaStream_t st, long long *launches, long long *acc_hi, bool prezeroed)
{
    if (n_rp_max <= 0 || ns_max <= 0) return cudaSuccess;
    BnlArgs a{};
    a.d_nrp = d_nrp;
    a.d_nsp = d_nsp;
    a.rkeys = rkeys;
    a.skeys = skeys;
    a.svals = svals;
    a.extreme = extreme;
    a.one = 1u;
    a.shape = shape;
    a.prezeroed = prezeroed;
    a.acc = acc;
    a.cnt = cnt;
    a.acc_hi = (agg == SUM || agg == AVG) && vb == 8 ? acc_hi : nullptr;
    const bool noval = agg == COUNT || agg == EXISTS || agg == NOT_EXISTS;
    const int v = noval ? 0 : (vb == 8 ? 8 : 4);
    const int ag = agg == AVG ? SUM : (agg == NOT_EXISTS ? EXISTS : agg);
    cudaError_t e;
    if (kb == 4) {
        if (v == 0) e = bnl_family_u32_v0(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
        else if (v == 4) e = bnl_family_u32_v4(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
        else e = bnl_family_u32_v8(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
    } else {
        if (v == 0) e = bnl_family_u64_v0(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
        else if (v == 4) e = bnl_family_u64_v4(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
        else e = bnl_family_u64_v8(op, ag, a, n_rp_max, ns_max, scratch, num_sms, st);
    }
    ++*launches;
    return e;
}

}  // namespace ng
