// traj.cu -- trajectory-level results.
//
// The application of the paper asks for the stars that come within d of
// another star and the time intervals in which this happens; the
// search itself works on segments.  Here every segment-level result
// (q, l, [t_s, t_e]) is mapped to its trajectory pair (query_traj[q],
// entry_traj[l]) and the intervals of each pair are merged into the maximal
// connected pieces of their union (closed intervals that touch merge):
//   1. keys: t_start (order-preserving bits) and the pair (qt << 32 | et);
//   2. two stable LSD radix sorts: by t_start, then by pair;
//   3. group heads + exclusive scan -> one thread per pair group merges its
//      time-sorted intervals (groups hold at most a few hundred results);
//   4. exclusive scan of the merged counts -> compact output.
#include "internal.cuh"

namespace dts {
namespace {

constexpr int TB = 256;

inline unsigned blocks(size_t n) { return (unsigned)((n + TB - 1) / TB); }

__global__ void __launch_bounds__(TB) k_traj_keys(const dts_result* __restrict__ r, size_t n,
                                                 const uint32_t* __restrict__ qtraj, size_t nqid,
                                                 const uint32_t* __restrict__ etraj, size_t neid,
                                                 unsigned long long* __restrict__ tkey,
                                                 unsigned long long* __restrict__ pkey,
                                                 uint32_t* __restrict__ vals,
                                                 unsigned int* __restrict__ bad) {
    const size_t k = (size_t)blockIdx.x * TB + threadIdx.x;
    if (k >= n) return;
    const dts_result x = r[k];
    if (x.query_id >= nqid || x.entry_id >= neid) {
        atomicOr(bad, 1u);
        tkey[k] = 0;
        pkey[k] = 0;
    } else {
        tkey[k] = ordered_bits(x.t_start);
        pkey[k] = ((unsigned long long)__ldg(qtraj + x.query_id) << 32) |
                  __ldg(etraj + x.entry_id);
    }
    vals[k] = (uint32_t)k;
}

// pair keys re-gathered in t_start order (the second sort's input)
__global__ void __launch_bounds__(TB) k_gather_u64(const unsigned long long* __restrict__ in,
                                                  const uint32_t* __restrict__ idx, size_t n,
                                                  unsigned long long* __restrict__ out) {
    const size_t k = (size_t)blockIdx.x * TB + threadIdx.x;
    if (k < n) out[k] = in[idx[k]];
}

__global__ void __launch_bounds__(TB) k_heads(const unsigned long long* __restrict__ pkey,
                                             size_t n, uint32_t* __restrict__ head) {
    const size_t k = (size_t)blockIdx.x * TB + threadIdx.x;
    if (k < n) head[k] = (k == 0 || pkey[k] != pkey[k - 1]) ? 1u : 0u;
}

__global__ void __launch_bounds__(TB) k_group_starts(const uint32_t* __restrict__ head,
                                                    const uint32_t* __restrict__ gidx, size_t n,
                                                    uint32_t* __restrict__ gstart) {
    const size_t k = (size_t)blockIdx.x * TB + threadIdx.x;
    if (k < n && head[k]) gstart[gidx[k]] = (uint32_t)k;
    if (k == 0) gstart[gidx[n]] = (uint32_t)n;    // sentinel: number of groups -> n
}

// One thread per pair group: merge its t_start-sorted intervals.
__global__ void __launch_bounds__(TB) k_merge(const dts_result* __restrict__ r,
                                             const uint32_t* __restrict__ order,
                                             const unsigned long long* __restrict__ pkey,
                                             const uint32_t* __restrict__ gstart, uint32_t ng,
                                             dts_traj_result* __restrict__ tmp,
                                             uint32_t* __restrict__ gcount) {
    const uint32_t g = blockIdx.x * TB + threadIdx.x;
    if (g >= ng) return;
    const uint32_t a = gstart[g], b = gstart[g + 1];
    const unsigned long long key = pkey[a];
    uint32_t m = 0;
    dts_result x = r[order[a]];
    double lo = x.t_start, hi = x.t_end;
    for (uint32_t i = a + 1; i < b; ++i) {
        x = r[order[i]];
        if (x.t_start <= hi) {                  // touching or overlapping: same piece
            hi = fmax(hi, x.t_end);
        } else {
            tmp[a + m++] = dts_traj_result{(uint32_t)(key >> 32), (uint32_t)key, lo, hi};
            lo = x.t_start;
            hi = x.t_end;
        }
    }
    tmp[a + m++] = dts_traj_result{(uint32_t)(key >> 32), (uint32_t)key, lo, hi};
    gcount[g] = m;
}

__global__ void __launch_bounds__(TB) k_compact(const dts_traj_result* __restrict__ tmp,
                                               const uint32_t* __restrict__ gstart,
                                               const uint32_t* __restrict__ gcount,
                                               const unsigned long long* __restrict__ goff,
                                               uint32_t ng, dts_traj_result* __restrict__ out) {
    const uint32_t g = blockIdx.x * TB + threadIdx.x;
    if (g >= ng) return;
    const uint32_t a = gstart[g];
    for (uint32_t j = 0; j < gcount[g]; ++j) out[goff[g] + j] = tmp[a + j];
}

}  // namespace

void merge_trajectories_device(const dts_result* r, size_t n, const uint32_t* qtraj,
                               size_t nqid, const uint32_t* etraj, size_t neid,
                               cudaStream_t s, dts_traj_result** out, size_t* count) {
    *out = nullptr;
    *count = 0;
    if (n == 0) return;
    if (n >= (size_t(1) << 32)) throw Error(DTS_ENOTSUP, "more than 2^32 results to merge");
    DevBuf<unsigned long long> tkey(n, s), pkey(n, s), k2(n, s), pk_sorted(n, s);
    DevBuf<uint32_t> order(n, s), v2(n, s);
    DevBuf<unsigned int> bad(1, s);
    DTS_CUDA(cudaMemsetAsync(bad.p, 0, sizeof(unsigned int), s));
    k_traj_keys<<<blocks(n), TB, 0, s>>>(r, n, qtraj, nqid, etraj, neid, tkey.p, pkey.p, order.p,
                                         bad.p);
    DTS_LAUNCH_CHECK();
    // stable: by t_start, then by (query_traj, entry_traj)
    radix_sort_pairs(tkey.p, order.p, k2.p, v2.p, n, 64, s);
    k_gather_u64<<<blocks(n), TB, 0, s>>>(pkey.p, order.p, n, pk_sorted.p);
    DTS_LAUNCH_CHECK();
    radix_sort_pairs(pk_sorted.p, order.p, k2.p, v2.p, n, 64, s);
    // groups of equal pair keys
    DevBuf<uint32_t> head(n, s), gidx(n + 1, s);
    k_heads<<<blocks(n), TB, 0, s>>>(pk_sorted.p, n, head.p);
    DTS_LAUNCH_CHECK();
    scan_exclusive_u32_to_u32(head.p, gidx.p, n, s);
    unsigned int hbad = 0;
    uint32_t ng = 0;
    DTS_CUDA(cudaMemcpyAsync(&ng, gidx.p + n, sizeof(ng), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaMemcpyAsync(&hbad, bad.p, sizeof(hbad), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    if (hbad) throw Error(DTS_EINVAL, "a result id is outside query_traj / entry_traj");
    DevBuf<uint32_t> gstart(ng + 1, s), gcount(ng, s);
    DevBuf<unsigned long long> goff(ng + 1, s);
    DevBuf<dts_traj_result> tmp(n, s);
    k_group_starts<<<blocks(n), TB, 0, s>>>(head.p, gidx.p, n, gstart.p);
    DTS_LAUNCH_CHECK();
    k_merge<<<blocks(ng), TB, 0, s>>>(r, order.p, pk_sorted.p, gstart.p, ng, tmp.p, gcount.p);
    DTS_LAUNCH_CHECK();
    scan_exclusive_u32_to_u64(gcount.p, goff.p, ng, s);
    unsigned long long total = 0;
    DTS_CUDA(cudaMemcpyAsync(&total, goff.p + ng, sizeof(total), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    dts_traj_result* o = static_cast<dts_traj_result*>(cache_alloc(total * sizeof(dts_traj_result)));
    k_compact<<<blocks(ng), TB, 0, s>>>(tmp.p, gstart.p, gcount.p, goff.p, ng, o);
    DTS_LAUNCH_CHECK();
    DTS_CUDA(cudaStreamSynchronize(s));
    *out = o;
    *count = (size_t)total;
}

}  // namespace dts
