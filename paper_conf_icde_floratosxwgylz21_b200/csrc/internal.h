// internal.h -- host-side declarations shared by the C-ABI implementation
// (api.cpp) and the kernel launchers (k_*.cu).  Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

struct nestgpu_ctx;

namespace ng {

// Per-device launch setup cache (api.cpp).  The opt-in to more than 48 KB of
// dynamic shared memory (cudaFuncSetAttribute) and the occupancy a launcher
// sizes its persistent grid from are per DEVICE, so a process driving several
// GPUs (one context per device) must not reuse the first device's setup.
// Entries are keyed by (kernel, key, device) and guarded by a mutex.
bool launch_cache_get(const void *kernel, long long key, int dev, int *value);
void launch_cache_put(const void *kernel, long long key, int dev, int value);

// *value = the cached setup of `kernel` for `key` on the current device, or
// init(dev, value) once (cudaFuncSetAttribute + occupancy; it may run twice
// when two threads race, which is harmless: both calls are idempotent).
template <typename F>
inline cudaError_t per_device_setup(const void *kernel, long long key, int *value, F init)
{
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (launch_cache_get(kernel, key, dev, value)) return cudaSuccess;
    if ((e = init(dev, value)) != cudaSuccess) return e;
    launch_cache_put(kernel, key, dev, *value);
    return cudaSuccess;
}

// Context accessors (api.cpp) for host-side modules such as cost.cpp.
void *ctx_scratch_alloc(nestgpu_ctx *c, size_t bytes);   // nullptr when the arena is exhausted
void ctx_scratch_reset(nestgpu_ctx *c);
cudaStream_t ctx_stream(nestgpu_ctx *c);
int ctx_num_sms(nestgpu_ctx *c);
long long *ctx_launches(nestgpu_ctx *c);
unsigned *ctx_pinned(nestgpu_ctx *c);
int ctx_device(nestgpu_ctx *c);
int32_t ctx_fail(nestgpu_ctx *c, int32_t code, const char *msg);

// out[i] = hash(seed, i) % mod (+ lo), for synthetic calibration inputs; w = 4 or 8.
cudaError_t launch_fill_hash(void *out, int w, long long n, unsigned seed, unsigned long long mod, long long lo,
                             cudaStream_t st, long long *launches);
// out[i] = lo + i / div (ascending runs), w = 4 or 8.
cudaError_t launch_fill_runs(void *out, int w, long long n, long long div, long long lo, cudaStream_t st,
                             long long *launches);

// Every launcher returns the cudaError_t of its launch(es) and bumps *launches
// by the number of kernels it launched.
//
// Small scratch regions (counters, look-back status words, tile offsets) of
// one public call are zeroed by ONE fill kernel before its first launch
// instead of one cudaMemsetAsync per launcher (each a separate GPU operation
// on the latency path of small queries); launchers given prezeroed = true
// skip their own memsets -- the caller has put every region they need
// (see the *_zero_bytes helpers) on the fill list.
struct FillList {
    int n = 0;
    void *p[24];
    unsigned long long bytes[24];
    unsigned long long pat[24];   // byte value replicated, or (word) a 64-bit pattern
    unsigned char word[24];       // 1: 8-byte pattern (8-B aligned region, bytes % 8 == 0)
    bool add(void *ptr, size_t b, unsigned char v = 0)
    {
        if (!ptr || !b) return true;
        if (n >= 24) return false;
        p[n] = ptr;
        bytes[n] = b;
        pat[n] = 0x0101010101010101ull * v;
        word[n] = 0;
        n++;
        return true;
    }
    bool add_words(void *ptr, size_t b, unsigned long long v)
    {
        if (!ptr || !b) return true;
        if (n >= 24) return false;
        p[n] = ptr;
        bytes[n] = b;
        pat[n] = v;
        word[n] = 1;
        n++;
        return true;
    }
};
cudaError_t launch_fill(const FillList &f, cudaStream_t st, long long *launches);
// scratch bytes a prezeroed launcher expects zero (regions start at scratch)
size_t filter_zero_bytes(long long n, bool ordered);
size_t finalize_scratch_bytes(long long n);
size_t finalize_zero_bytes();   // the part of the finalize scratch that must be zero

// a2 / a3: filter rows [0, n) by `preds`, compact survivors in row order.
//   out_ids    : int32 row ids of survivors (nullable)
//   out_keys   : encoded keys (K = uint32 when kb == 4, uint64 when 8) (nullable)
//   out_kvalid : 1 byte per survivor, key not NULL (nullable)
//   out_vals   : payload (vb = 4 or 8 bytes; nullable)
//   drop_null_key / drop_null_val : NULL key / payload rows do not survive
//   keymask    : if non-null, [0] &= and [1] |= every survivor's encoded key
//                (radix digits where they agree need no sort pass)
//   extreme    : if non-null, [0] |= any survivor payload == max of its type,
//                [1] |= any == min (for the MIN/MAX identity check),
//                (u64)[2..3] = max |payload| (atomicMax; 32-bit partial sums)
//   scratch    : tile status + counter, from filter_scratch_bytes(n)
//   out_count  : int64 survivor count (device)
//   ordered_phase: 0 = one call (ordered iff out_ids); 1 / 2 = the two
//     halves of an ordered filter without row ids: 1 counts + scans (the
//     caller reads *out_count and sizes the outputs), 2 writes the outputs
//     (same arguments and scratch; drop_null_* must be 0)
size_t filter_scratch_bytes(long long n);
cudaError_t launch_filter(long long n, const PredSet &preds, const KeySrc &key, int kb,
                          const ValSrc &val, int vb, int drop_null_key, int drop_null_val,
                          int *out_ids, void *out_keys, uint8_t *out_kvalid, void *out_vals,
                          unsigned long long *keymask, unsigned *extreme, void *scratch,
                          long long *out_count, cudaStream_t st, long long *launches, bool prezeroed = false,
                          int ordered_phase = 0);

// a4: histograms of the digits at `shifts` (np of them) over n encoded keys,
// and their exclusive scans into digit_base[np][256].
//   rb: digit bits (8 or 9); hist / digit_base hold np * 2^rb words
// hist: hist_bytes() of scratch (8 x 512 bins + a CTA-done counter); the
// kernel's last CTA scans the bins into digit_base (one launch).
size_t hist_bytes();
//   encx: XOR applied to every key read (encodes a raw signed key column)
cudaError_t launch_digit_hist(int kb, const void *keys, long long n, const int *shifts, int np, unsigned *hist,
                              unsigned *digit_base, int num_sms, cudaStream_t st, long long *launches, int rb = 8,
                              bool prezeroed = false, unsigned long long encx = 0);

// a4: one stable LSD radix pass on the rb-bit digit (rb = 8 or 9) at bit
// `shift` of the encoded keys.
//   digit_base: 2^rb uint32 global exclusive offsets of the digit (device)
size_t sort_scratch_bytes(long long n);
cudaError_t launch_radix_pass(int kb, int vb, const void *kin, void *kout, const void *vin, void *vout,
                              long long n, int shift, const unsigned *digit_base, void *scratch,
                              cudaStream_t st, long long *launches, int rb = 8);
// The same with different key widths in and out: 8 -> 4 drops the high word
// (all keys must share it), 4 -> 8 re-attaches `hi` as the high word.
cudaError_t launch_radix_pass_x(int kb_in, int kb_out, int vb, const void *kin, void *kout, const void *vin,
                                void *vout, long long n, int shift, const unsigned *digit_base, void *scratch,
                                unsigned hi, cudaStream_t st, long long *launches, int rb = 8,
                                bool prezeroed = false, unsigned long long encx = 0);
// scratch bytes of one radix pass that must be zero (per-tile digit counts + counter)
size_t sort_pass_zero_bytes(long long n, int kb, int vb, int rb);

// a4 (large S'): two-round-trip MSD bucket sort (k_bsort.cu).
//   bsort_capacity: largest bucket the finish kernel sorts in shared memory
//   launch_bsort_hist: group histograms of the D-bit digit at s1 (nb = 2^D
//     <= 4096 buckets), scanned into per-group starts (hscratch,
//     bsort_hist_bytes), bucket bases base[0..nb] and the largest bucket
//     *maxb (device); zscratch (bsort_zero_bytes) must be zero
//   launch_bsort_sort: partition kin -> kmid (kb_in -> kb_mid key bytes) by
//     the D-bit digit, then finish each bucket kmid -> kout (kb_mid ->
//     kb_out; 4 -> 8 re-attaches hi) over the np2 <= 6-bit digit windows
//     (pshift, pbits); valid only when *maxb <= bsort_capacity(kb_mid, vb)
int bsort_capacity(int kb_mid, int vb);
size_t bsort_hist_bytes(long long n, int nb);
size_t bsort_zero_bytes(int nb);
cudaError_t launch_bsort_hist(int kb_in, const void *keys, long long n, int s1, int nb, void *hscratch,
                              unsigned *zscratch, unsigned *base, unsigned *maxb, cudaStream_t st, long long *launches);
cudaError_t launch_bsort_sort(int kb_in, int kb_mid, int kb_out, int vb, const void *kin, const void *vin,
                              void *kmid, void *vmid, void *kout, void *vout, long long n, int s1, int D,
                              const int *pshift, const int *pbits, int np2, const void *hscratch,
                              const unsigned *base, unsigned hi, cudaStream_t st, long long *launches);

// Partial aggregates per R' tuple: acc (int64) + cnt (int64); identity init.
// n: host upper bound (grid size); d_n: the actual count (device)
cudaError_t launch_init_partials(long long n, const long long *d_n, int agg, long long *acc, long long *cnt,
                                 cudaStream_t st, long long *launches);

// a5 + a6: per R' tuple binary search of the sorted index and fold of the
// qualifying range(s).  d_nrp: device count of R'.  Long ranges go to a
// warp-per-range second kernel.
size_t range_scratch_bytes(long long n_rp_max);
// Indexes of at most this many entries: every range is folded inline by its
// thread (no long-range kernel) and the keys themselves serve as the search
// samples (no sample kernel) -- fewer launches for small, latency-bound
// queries.
constexpr long long RANGE_INLINE_MAX = 4096;
//   pre / suf: optional prefix / suffix aggregates of the index payload
//   (launch_index_aux); non-equality and SUM/AVG ranges are then O(1).
//   pre_hi / acc_hi: exact SUM of 64-bit payloads (nullable): pre holds the
//   prefix sums of the payloads' low 32-bit halves (unsigned) and pre_hi of
//   their high halves (signed), neither of which can overflow; a range's two
//   partial sums go to acc / acc_hi and finalize combines them in int128.
cudaError_t launch_range_agg(int kb, int vb, int op, int agg, long long n_rp_max, const long long *d_nrp,
                             const void *rkeys, const void *skeys, const void *svals, long long ns,
                             const long long *pre, const long long *suf, long long *acc, long long *cnt,
                             void *scratch, cudaStream_t st, long long *launches,
                             const long long *pre_hi = nullptr, long long *acc_hi = nullptr, bool prezeroed = false);

// Index-pruned evaluation (NEXT 3): pre[0..n] / suf[0..n] aggregates (MIN,
// MAX: both; SUM: pre only) of the co-sorted payload of an index.
size_t index_aux_scratch_bytes(long long n);
// '=' MIN/MAX: per-key group aggregates grp[p] = AGG(payload[run start .. p])
// over the sorted index (segmented scan; runs of equal keys); n entries.
cudaError_t launch_index_group_agg(int agg, int kb, int vb, const void *keys, const void *payload, long long n,
                                   long long *grp, void *scratch, cudaStream_t st, long long *launches);
//   pre_hi (SUM only, nullable): split prefix sums -- pre over the low 32-bit
//   halves of the payload (unsigned), pre_hi over the high halves (signed).
cudaError_t launch_index_aux(int agg, int vb, const void *payload, long long n, long long *pre, long long *suf,
                             void *scratch, cudaStream_t st, long long *launches, long long *pre_hi = nullptr);

// a7: tiled block-nested-loop over R' x S'.  d_nrp / d_nsp: device counts.
size_t bnl_scratch_bytes(long long n_rp_max);
cudaError_t launch_bnl(int kb, int vb, int op, int agg, long long n_rp_max, const long long *d_nrp,
                       const void *rkeys, long long ns_max, const long long *d_nsp, const void *skeys,
                       const void *svals, const unsigned *extreme, long long *acc, long long *cnt,
                       void *scratch, int num_sms, int shape /* 0 auto, 1 full, 2 warp-split */,
                       cudaStream_t st, long long *launches, long long *acc_hi = nullptr, bool prezeroed = false);
//   acc_hi (SUM/AVG of 64-bit payloads, nullable, zeroed by the caller): exact
//   split accumulation -- acc += low 32-bit halves, acc_hi += high halves.

// Caching: R' positions 0..n-1; distinct keys of a sorted key run
// and the map R' position -> distinct id.
cudaError_t launch_iota(int *out, long long n, cudaStream_t st, long long *launches);
size_t group_scratch_bytes(long long n);
cudaError_t launch_group(int kb, const void *sorted_keys, const int *sorted_pos, long long n, void *uniq_keys, int *map,
                         long long *d_u, void *scratch, cudaStream_t st, long long *launches);

// a8 + a9: aggregate finalize, outer comparison, ordered compaction.
struct FinalizeArgs {
    long long n_rp_max;
    const long long *d_nrp;
    const int *ids;          // R' row ids
    const int *map;          // R' position -> partial-aggregate slot (nullable = identity)
    const uint8_t *kvalid;   // R' key not NULL (nullable = all valid)
    const long long *acc, *cnt;
    const long long *acc_hi;         // split SUM (nullable): sum = acc_hi * 2^32 + (u64)acc, exact in int128
    unsigned long long *overflow;    // set when a split SUM leaves int64 (reading R5 -> NESTGPU_ERR_OVERFLOW)
    const void *x_col;       // outer comparison column (nullable for EXISTS)
    const uint8_t *x_valid;
    int x_w;
    int agg, outer_op;
    long long a, b;
    long long row_id_base;
    int emit_all;
    long long *out_ids, *out_vals, *out_sum, *out_cnt;  // sum/cnt: AVG only (nullable)
    uint8_t *out_valid, *out_passed;
    long long *out_count;
    void *scratch;           // filter_scratch_bytes(n_rp_max)
};
cudaError_t launch_finalize(const FinalizeArgs &a, cudaStream_t st, long long *launches, bool prezeroed = false);

// Tiny queries (k_finalize.cu): the nested-loop strategy's whole sequence in
// one launch of one CTA when |S| <= TINY_S_MAX, |R| <= TINY_R_MAX and
// |R| x |S| <= TINY_PAIRS_MAX.  f: the finalize arguments (outputs,
// out_count = counts + 2, overflow unused); counts[0] |R'|, [1] |S'|, [8]
// overflow flag are written by the kernel.
// counts must have 128 + 8 * TINY_G_MAX bytes (the launcher zeroes them;
// the tail holds the per-CTA emit counts).
constexpr long long TINY_S_MAX = 4096, TINY_R_MAX = 4096, TINY_PAIRS_MAX = 1ll << 21;
constexpr int TINY_G_MAX = 256;
struct TinyArgs {
    long long nR, nS;
    PredSet rp, sp;
    KeySrc rk, sk;
    ValSrc v;
    int corr_op;
    int chunk;                      // outer tuples per CTA (set by the launcher)
    FinalizeArgs f;
    long long *counts;
    unsigned long long *status;     // counts + 16: per-CTA emit counts
};
cudaError_t launch_tiny_exec(const TinyArgs &t, int num_sms, cudaStream_t st, long long *launches);

// Survivor rows into a (peer) window: win_ids[off + i] = ids[i],
// win_vals[off + i] = vals[i], i < n; ends with __threadfence_system.
cudaError_t launch_put_rows(const long long *ids, const long long *vals, long long n, long long *win_ids,
                            long long *win_vals, cudaStream_t st, long long *launches);

// out[i] = src[ids[i] - base] (w = 4 or 8 bytes per value).
cudaError_t launch_gather(int w, const void *src, const long long *ids, long long n, long long base, void *out,
                          cudaStream_t st, long long *launches);

// Type-J two-level arrays, k_collect.cu.
//   bounds: per R' tuple the qualifying runs of the index, lens[i], int64
//   row_ids[i] (+ base), offsets[0..n] = exclusive prefix of lens, *total =
//   offsets[n] (all device).
//   fill  : values[e] = payload of slot e (widened), owner[e] = its row id.
size_t collect_scratch_bytes(long long n_rp_max);
cudaError_t launch_collect_bounds(int kb, int op, long long n_rp_max, const long long *d_nrp, const int *ids,
                                  const void *rkeys, const uint8_t *rkvalid, const void *skeys, long long ns,
                                  long long base, void *scratch, long long *lens, long long *row_ids,
                                  long long *offsets, long long *total, cudaStream_t st, long long *launches);
cudaError_t launch_collect_fill(int vb, const long long *d_nrp, const long long *offsets, const void *scratch,
                                const long long *row_ids, const void *payload, long long total, long long *values,
                                long long *owner, cudaStream_t st, long long *launches);
// IN over a two-level array: cnt[i] = x(row_ids[i]-base) in list i; ids32[i] = row_ids[i] - base.
cudaError_t launch_in_list(long long n, const long long *row_ids, const long long *offsets, const long long *values,
                           const void *x_col, int x_w, const uint8_t *x_valid, long long base, int *ids32,
                           long long *cnt, cudaStream_t st, long long *launches);
// out = (int32|int64) src with validity; *bad += valid values outside int32 (w == 4).
cudaError_t launch_materialize(int w, const long long *src, const uint8_t *valid_in, long long n, void *out,
                               uint8_t *valid_out, unsigned long long *bad, cudaStream_t st, long long *launches);

}  // namespace ng
