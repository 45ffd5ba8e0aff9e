// ooc.cu -- an entry database larger than the device budget
// (dts_index_params.mem_budget_bytes; SURVEY.md §8(e) fallback; the paper
// partitions D across GPU-equipped nodes so that aggregate GPU memory is
// large).
//
// D is split by t_start range into K temporal shards, each small enough to be
// indexed within the budget.  Each entry lives in exactly one shard; a query
// can only match entries of the shards it overlaps strictly in time, so the
// per-shard result
// sets are disjoint and their union is exact -- no deduplication.  (Routing
// uses each shard's exact min t_start and max t_end: q is sent to shard k iff
// q.t_end > t0min_k and q.t_start < t1max_k.)  The shards
// stay in pinned host memory; a search streams them through the device one
// after another (H2D, index build, routed queries, search with global ids)
// and one device sort restores the canonical (query id, entry id) order.
//
// Every pass over D runs in the kernels below (bounds + validation, a
// t_start histogram that fixes the shard boundaries and sizes exactly, the
// partition); the host only picks boundaries from the histogram and moves
// pinned chunks.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "internal.cuh"

namespace dts {
namespace {

constexpr int OT = 256;
constexpr int HBINS = 1 << 16;         // t_start histogram resolution

inline unsigned oblocks(size_t n) { return (unsigned)((n + OT - 1) / OT); }

// Validation (finite values, t_end >= t_start) and the t_start range, as
// order-preserving integer images (atomicMin / atomicMax).
__global__ void __launch_bounds__(OT) k_ooc_bounds(const double4* __restrict__ D, size_t n,
                                                  unsigned long long* __restrict__ tmm,
                                                  unsigned int* __restrict__ bad) {
    const size_t i = (size_t)blockIdx.x * OT + threadIdx.x;
    unsigned long long lo = ~0ull, hi = 0ull;
    if (i < n) {
        const double4 s0 = D[2 * i], s1 = D[2 * i + 1];
        const double c[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
        bool ok = true;
#pragma unroll
        for (int k = 0; k < 8; ++k) ok = ok && isfinite(c[k]);
        if (!ok) atomicOr(bad, 1u);
        else if (s1.x < s0.x) atomicOr(bad, 2u);
        else { lo = ordered_bits(s0.x); hi = lo; }
    }
    for (int o = 16; o; o >>= 1) {
        const unsigned long long a = __shfl_xor_sync(0xffffffffu, lo, o);
        const unsigned long long b = __shfl_xor_sync(0xffffffffu, hi, o);
        lo = a < lo ? a : lo;
        hi = b > hi ? b : hi;
    }
    if ((threadIdx.x & 31) == 0 && lo <= hi) {
        atomicMin(&tmm[0], lo);
        atomicMax(&tmm[1], hi);
    }
}

__device__ __forceinline__ int hist_bin(double t, double tmin, double inv) {
    const double f = floor((t - tmin) * inv);
    if (!(f > 0.0)) return 0;
    if (f >= (double)(HBINS - 1)) return HBINS - 1;
    return (int)f;
}

__global__ void __launch_bounds__(OT) k_ooc_hist(const double4* __restrict__ D, size_t n,
                                                double tmin, double inv,
                                                unsigned long long* __restrict__ hist) {
    const size_t i = (size_t)blockIdx.x * OT + threadIdx.x;
    if (i < n) atomicAdd(&hist[hist_bin(D[2 * i].x, tmin, inv)], 1ull);
}

// Shard of each row (by histogram bin: shard k = bins [edge[k], edge[k+1])).
// Counting pass (base == NULL): rows per shard and each shard's exact
// [min t_start, max t_end]; scatter pass: rows into a staging buffer grouped
// by shard (arrival order inside a shard; the final sort restores canonical
// order), with the global entry id and trajectory id.
__global__ void __launch_bounds__(OT) k_ooc_partition(const double4* __restrict__ D, size_t n,
                                                     size_t row0, double tmin, double inv,
                                                     const int* __restrict__ edge, int K,
                                                     const uint32_t* __restrict__ ids_in,
                                                     const uint32_t* __restrict__ traj_in,
                                                     unsigned long long* __restrict__ cursor,
                                                     const unsigned long long* __restrict__ base,
                                                     double4* __restrict__ Dout,
                                                     uint32_t* __restrict__ ids_out,
                                                     uint32_t* __restrict__ traj_out,
                                                     unsigned long long* __restrict__ tspan) {
    const size_t i = (size_t)blockIdx.x * OT + threadIdx.x;
    if (i >= n) return;
    const double4 s0 = D[2 * i], s1 = D[2 * i + 1];
    const int b = hist_bin(s0.x, tmin, inv);
    int k = 0;
    while (k + 1 < K && b >= edge[k + 1]) ++k;
    const unsigned long long c = atomicAdd(&cursor[k], 1ull);
    if (!base) {                          // counting pass: sizes and time span
        atomicMin(&tspan[2 * k], ordered_bits(s0.x));
        atomicMax(&tspan[2 * k + 1], ordered_bits(s1.x));
        return;
    }
    const unsigned long long pos = base[k] + c;
    Dout[2 * pos] = s0;
    Dout[2 * pos + 1] = s1;
    ids_out[pos] = ids_in ? ids_in[i] : (uint32_t)(row0 + i);
    if (traj_out) traj_out[pos] = traj_in[i];
}

// Queries that can overlap shard k strictly in time.
__global__ void __launch_bounds__(OT) k_ooc_route(const double4* __restrict__ Q, uint32_t nq,
                                                 double t_lo, double t_hi,
                                                 uint32_t* __restrict__ flag) {
    const uint32_t i = blockIdx.x * OT + threadIdx.x;
    if (i >= nq) return;
    const double q0 = Q[2 * (size_t)i].x, q1 = Q[2 * (size_t)i + 1].x;
    flag[i] = (q1 > t_lo && q0 < t_hi) ? 1u : 0u;
}

__global__ void __launch_bounds__(OT) k_ooc_gather_q(const double4* __restrict__ Q, uint32_t nq,
                                                    const uint32_t* __restrict__ flag,
                                                    const uint32_t* __restrict__ pos,
                                                    const uint32_t* __restrict__ qmap,
                                                    uint32_t qid_base,
                                                    const uint32_t* __restrict__ qtraj,
                                                    double4* __restrict__ Qk,
                                                    uint32_t* __restrict__ mapk,
                                                    uint32_t* __restrict__ trajk,
                                                    uint32_t* __restrict__ rowk) {
    const uint32_t i = blockIdx.x * OT + threadIdx.x;
    if (i >= nq || !flag[i]) return;
    const uint32_t j = pos[i];
    Qk[2 * (size_t)j] = Q[2 * (size_t)i];
    Qk[2 * (size_t)j + 1] = Q[2 * (size_t)i + 1];
    mapk[j] = qmap ? qmap[i] : qid_base + i;
    if (trajk) trajk[j] = qtraj[i];
    if (rowk) rowk[j] = i;
}

// counts[row of Q] += per-shard counts (count-only search).
__global__ void __launch_bounds__(OT) k_ooc_add_counts(const uint32_t* __restrict__ ck,
                                                      const uint32_t* __restrict__ rowk,
                                                      uint32_t n, uint32_t* __restrict__ counts) {
    const uint32_t j = blockIdx.x * OT + threadIdx.x;
    if (j < n) counts[rowk[j]] += ck[j];      // rows are distinct within a shard
}

}  // namespace

// Device bytes one index build + search over n entries may hold at once: the
// 68-byte records and ids, the 8-cell block hash (<= 3.3 x 32 B per entry in
// the worst case of one block per entry), the build's packed keys (2 x 8 B)
// and the device copy of D (64 B) -- about 310 B per entry.
uint64_t index_bytes_estimate(size_t n) { return (uint64_t)n * 310ull + (64ull << 20); }

void ooc_build(dts_index* idx, const dts_segment* D, size_t n, const dts_index_params& p,
               cudaStream_t s) {
    const uint64_t budget = p.mem_budget_bytes;
    OocIndex* o = new OocIndex();
    idx->ooc = o;
    idx->n = n;
    o->p = p;
    o->p.mem_budget_bytes = 0;
    o->p.entry_ids = nullptr;
    o->p.entry_traj = nullptr;
    const int K0 = (int)std::min<uint64_t>(
        4096, std::max<uint64_t>(2, (index_bytes_estimate(n) + budget - 1) / std::max<uint64_t>(budget, 1) + 1));
    // chunks of D through the device: a quarter of the budget for the chunk
    // and its staging copy
    const size_t chunk = std::max<size_t>(1 << 14, std::min<size_t>(n, budget / 4 / 160));
    DevBuf<dts_segment> dch(chunk, s), dout(chunk, s);
    DevBuf<uint32_t> dids(p.entry_ids ? chunk : 0, s), dtraj(p.entry_traj ? chunk : 0, s);
    DevBuf<uint32_t> oids(chunk, s), otraj(p.entry_traj ? chunk : 0, s);
    DevBuf<unsigned long long> tmm(2, s), hist(HBINS, s);
    DevBuf<unsigned int> bad(1, s);
    unsigned long long init[2] = {~0ull, 0ull};
    DTS_CUDA(cudaMemcpyAsync(tmm.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    DTS_CUDA(cudaMemsetAsync(bad.p, 0, sizeof(unsigned int), s));
    // pass 1: validation + t_start range
    for (size_t a = 0; a < n; a += chunk) {
        const size_t m = std::min(chunk, n - a);
        DTS_CUDA(cudaMemcpyAsync(dch.p, D + a, m * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
        k_ooc_bounds<<<oblocks(m), OT, 0, s>>>(reinterpret_cast<const double4*>(dch.p), m, tmm.p,
                                               bad.p);
        DTS_LAUNCH_CHECK();
    }
    unsigned long long ht[2];
    unsigned int hbad = 0;
    DTS_CUDA(cudaMemcpyAsync(ht, tmm.p, sizeof(ht), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaMemcpyAsync(&hbad, bad.p, sizeof(hbad), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    if (hbad & 1) throw Error(DTS_EINVAL, "entry segment with a non-finite coordinate or time");
    if (hbad & 2) throw Error(DTS_EINVAL, "entry segment with t_end < t_start");
    const double tmin = from_ordered_bits(ht[0]), tmax = from_ordered_bits(ht[1]);
    const double inv = tmax > tmin ? (double)HBINS / (tmax - tmin) : 0.0;
    // pass 2: t_start histogram -> shard edges (histogram bins) and sizes
    DTS_CUDA(cudaMemsetAsync(hist.p, 0, HBINS * sizeof(unsigned long long), s));
    for (size_t a = 0; a < n; a += chunk) {
        const size_t m = std::min(chunk, n - a);
        DTS_CUDA(cudaMemcpyAsync(dch.p, D + a, m * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
        k_ooc_hist<<<oblocks(m), OT, 0, s>>>(reinterpret_cast<const double4*>(dch.p), m, tmin, inv,
                                             hist.p);
        DTS_LAUNCH_CHECK();
    }
    std::vector<unsigned long long> hh(HBINS);
    DTS_CUDA(cudaMemcpyAsync(hh.data(), hist.p, HBINS * sizeof(unsigned long long),
                             cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    std::vector<int> edge{0};
    std::vector<size_t> size;
    {
        const double target = (double)n / K0;
        unsigned long long acc = 0;
        for (int b = 0; b < HBINS; ++b) {
            acc += hh[b];
            if (acc >= target * (double)(edge.size()) && b + 1 < HBINS && (int)edge.size() < K0 &&
                acc < n) {
                edge.push_back(b + 1);
            }
        }
        for (size_t k = 0; k < edge.size(); ++k) {
            const int b0 = edge[k], b1 = k + 1 < edge.size() ? edge[k + 1] : HBINS;
            unsigned long long c = 0;
            for (int b = b0; b < b1; ++b) c += hh[b];
            size.push_back((size_t)c);
        }
    }
    const int K = (int)edge.size();
    o->off.assign(K + 1, 0);
    for (int k = 0; k < K; ++k) o->off[k + 1] = o->off[k] + size[k];
    o->shards.resize(K);
    for (int k = 0; k < K; ++k) o->shards[k].n = size[k];
    // pass 3: partition into pinned per-shard storage
    DTS_CUDA(cudaMallocHost(&o->D_h, std::max<size_t>(n, 1) * sizeof(dts_segment)));
    DTS_CUDA(cudaMallocHost(&o->ids_h, std::max<size_t>(n, 1) * sizeof(uint32_t)));
    if (p.entry_traj) DTS_CUDA(cudaMallocHost(&o->traj_h, n * sizeof(uint32_t)));
    DevBuf<int> dedge(K, s);
    DevBuf<unsigned long long> cursor(K, s), cbase(K, s), tspan(2 * K, s);
    DTS_CUDA(cudaMemcpyAsync(dedge.p, edge.data(), K * sizeof(int), cudaMemcpyHostToDevice, s));
    {
        std::vector<unsigned long long> init(2 * K);
        for (int k = 0; k < K; ++k) { init[2 * k] = ~0ull; init[2 * k + 1] = 0ull; }
        DTS_CUDA(cudaMemcpyAsync(tspan.p, init.data(), 2 * K * 8, cudaMemcpyHostToDevice, s));
        DTS_CUDA(cudaStreamSynchronize(s));
    }
    std::vector<unsigned long long> filled(K, 0), ccount(K), cb(K);
    for (size_t a = 0; a < n; a += chunk) {
        const size_t m = std::min(chunk, n - a);
        DTS_CUDA(cudaMemcpyAsync(dch.p, D + a, m * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
        if (p.entry_ids)
            DTS_CUDA(cudaMemcpyAsync(dids.p, p.entry_ids + a, m * 4, cudaMemcpyHostToDevice, s));
        if (p.entry_traj)
            DTS_CUDA(cudaMemcpyAsync(dtraj.p, p.entry_traj + a, m * 4, cudaMemcpyHostToDevice, s));
        // count this chunk's rows per shard, then scatter them grouped by
        // shard at the chunk's exclusive-scan bases
        DTS_CUDA(cudaMemsetAsync(cursor.p, 0, K * sizeof(unsigned long long), s));
        k_ooc_partition<<<oblocks(m), OT, 0, s>>>(
            reinterpret_cast<const double4*>(dch.p), m, a, tmin, inv, dedge.p, K, dids.p,
            dtraj.p, cursor.p, nullptr, reinterpret_cast<double4*>(dout.p), oids.p, otraj.p,
            tspan.p);
        DTS_LAUNCH_CHECK();
        DTS_CUDA(cudaMemcpyAsync(ccount.data(), cursor.p, K * sizeof(unsigned long long),
                                 cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        unsigned long long acc = 0;
        for (int k = 0; k < K; ++k) { cb[k] = acc; acc += ccount[k]; }
        DTS_CUDA(cudaMemcpyAsync(cbase.p, cb.data(), K * sizeof(unsigned long long),
                                 cudaMemcpyHostToDevice, s));
        DTS_CUDA(cudaMemsetAsync(cursor.p, 0, K * sizeof(unsigned long long), s));
        k_ooc_partition<<<oblocks(m), OT, 0, s>>>(
            reinterpret_cast<const double4*>(dch.p), m, a, tmin, inv, dedge.p, K, dids.p,
            dtraj.p, cursor.p, cbase.p, reinterpret_cast<double4*>(dout.p), oids.p, otraj.p,
            tspan.p);
        DTS_LAUNCH_CHECK();
        for (int k = 0; k < K; ++k) {
            if (!ccount[k]) continue;
            const size_t dst = o->off[k] + filled[k];
            DTS_CUDA(cudaMemcpyAsync(o->D_h + dst, dout.p + cb[k], ccount[k] * sizeof(dts_segment),
                                     cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaMemcpyAsync(o->ids_h + dst, oids.p + cb[k], ccount[k] * 4,
                                     cudaMemcpyDeviceToHost, s));
            if (p.entry_traj)
                DTS_CUDA(cudaMemcpyAsync(o->traj_h + dst, otraj.p + cb[k], ccount[k] * 4,
                                         cudaMemcpyDeviceToHost, s));
            filled[k] += ccount[k];
        }
        DTS_CUDA(cudaStreamSynchronize(s));
    }
    std::vector<unsigned long long> ts(2 * K);
    DTS_CUDA(cudaMemcpyAsync(ts.data(), tspan.p, 2 * K * 8, cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    for (int k = 0; k < K; ++k) {
        if (filled[k] != o->shards[k].n) throw Error(DTS_EINTERNAL, "temporal shard size mismatch");
        // exact routing bounds: an entry of shard k starts at or after t0min
        // and ends at or before t1max
        o->shards[k].t0min = filled[k] ? from_ordered_bits(ts[2 * k]) : 0.0;
        o->shards[k].t1max = filled[k] ? from_ordered_bits(ts[2 * k + 1]) : 0.0;
    }
    idx->eid_bits = 32;
}

void ooc_free(OocIndex* o) {
    if (!o) return;
    if (o->D_h) cudaFreeHost(o->D_h);
    if (o->ids_h) cudaFreeHost(o->ids_h);
    if (o->traj_h) cudaFreeHost(o->traj_h);
    delete o;
}

// Search (or count) of device Q against every shard in turn.  Results: the
// union in canonical order (device memory, cache_alloc'd); counts_out (device,
// count-only mode): per-query counts summed over the shards.
void ooc_search(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                uint32_t qid_base, cudaStream_t s, SearchOut* out, dts_search_stats* stats,
                const uint32_t* qmap, const uint32_t* qtraj, bool excl, bool count_only,
                uint32_t* counts_out) {
    const OocIndex* o = idx->ooc;
    out->results = nullptr;
    out->count = 0;
    dts_search_stats agg{};
    if (count_only && counts_out && nq)
        DTS_CUDA(cudaMemsetAsync(counts_out, 0, nq * sizeof(uint32_t), s));
    if (excl && !(qtraj && o->traj_h))
        throw Error(DTS_EINVAL, "exclude_same_trajectory needs query_traj and an index built "
                                "with entry_traj");
    std::vector<SearchOut> parts;
    unsigned long long total = 0;
    const double4* Q = reinterpret_cast<const double4*>(Q_dev);
    DevBuf<uint32_t> flag(nq, s), pos(nq + 1, s);
    try {
        for (size_t k = 0; k < o->shards.size() && nq; ++k) {
            const OocShard& sh = o->shards[k];
            if (sh.n == 0) continue;
            // the queries this shard can answer: strict overlap with an entry
            // needs q.t_end > its t_start >= t0min and q.t_start < its t_end
            // <= t1max (exact comparisons of stored values)
            k_ooc_route<<<oblocks(nq), OT, 0, s>>>(Q, (uint32_t)nq, sh.t0min, sh.t1max, flag.p);
            DTS_LAUNCH_CHECK();
            scan_exclusive_u32_to_u32(flag.p, pos.p, nq, s);
            uint32_t nqk = 0;
            DTS_CUDA(cudaMemcpyAsync(&nqk, pos.p + nq, 4, cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaStreamSynchronize(s));
            if (nqk == 0) continue;
            DevBuf<dts_segment> Qk(nqk, s);
            DevBuf<uint32_t> mapk(nqk, s), trajk(qtraj ? nqk : 0, s), rowk(count_only ? nqk : 0, s);
            k_ooc_gather_q<<<oblocks(nq), OT, 0, s>>>(Q, (uint32_t)nq, flag.p, pos.p, qmap, qid_base,
                                                      qtraj, reinterpret_cast<double4*>(Qk.p),
                                                      mapk.p, trajk.p, rowk.p);
            DTS_LAUNCH_CHECK();
            // the shard: pinned host -> device, index build with global ids
            DevBuf<dts_segment> Dk(sh.n, s);
            DevBuf<uint32_t> idk(sh.n, s), tk(o->traj_h ? sh.n : 0, s);
            DTS_CUDA(cudaMemcpyAsync(Dk.p, o->D_h + o->off[k], sh.n * sizeof(dts_segment),
                                     cudaMemcpyHostToDevice, s));
            DTS_CUDA(cudaMemcpyAsync(idk.p, o->ids_h + o->off[k], sh.n * 4, cudaMemcpyHostToDevice, s));
            if (tk.p)
                DTS_CUDA(cudaMemcpyAsync(tk.p, o->traj_h + o->off[k], sh.n * 4,
                                         cudaMemcpyHostToDevice, s));
            dts_index sub;
            sub.device = idx->device;
            dts_index_params sp = o->p;
            sp.entry_ids = idk.p;
            sp.entry_traj = tk.p;
            try {
                build_index_device(&sub, Dk.p, sh.n, sp, s);
                SearchOut so;
                dts_search_stats cs{};
                DevBuf<uint32_t> ck(count_only ? nqk : 0, s);
                search_device(&sub, Qk.p, nqk, d, 0, s, &so, &cs, ~0ull, mapk.p, trajk.p, excl,
                              count_only, ck.p);
                if (count_only && counts_out) {
                    k_ooc_add_counts<<<oblocks(nqk), OT, 0, s>>>(ck.p, rowk.p, nqk, counts_out);
                    DTS_LAUNCH_CHECK();
                }
                if (!count_only && so.count) parts.push_back(so);
                total += so.count;
                agg.candidates += cs.candidates;
                agg.cell_lookups += cs.cell_lookups;
                agg.max_results_per_query = std::max(agg.max_results_per_query,
                                                     cs.max_results_per_query);
                DTS_CUDA(cudaStreamSynchronize(s));
            } catch (...) {
                free_index_arrays(&sub);
                throw;
            }
            free_index_arrays(&sub);
        }
        if (!count_only && total) {
            // per-shard results are disjoint: concatenate, one device sort
            dts_result* fin = static_cast<dts_result*>(cache_alloc(total * sizeof(dts_result)));
            size_t at = 0;
            for (auto& pr : parts) {
                DTS_CUDA(cudaMemcpyAsync(fin + at, pr.results, pr.count * sizeof(dts_result),
                                         cudaMemcpyDeviceToDevice, s));
                at += pr.count;
            }
            DTS_CUDA(cudaStreamSynchronize(s));
            for (auto& pr : parts) cache_free(pr.results);
            parts.clear();
            try {
                canonicalize_device(fin, total, s);
            } catch (...) {
                cache_free(fin);
                throw;
            }
            out->results = fin;
        }
    } catch (...) {
        cudaStreamSynchronize(s);
        for (auto& pr : parts) cache_free(pr.results);
        throw;
    }
    out->count = (size_t)total;
    agg.results = total;
    if (stats) *stats = agg;
}

}  // namespace dts
