// search.cu -- the search hot path: query prep, fused candidate streaming +
// fp64 refinement in two passes (count, scatter), and canonical ordering.
//
// Paper (§IV): one GPU thread per query segment loops over a
// candidate set obtained from the index (GPUSpatial: U_k copied from A, Alg. 1
// l.9 P:L59; GPUTemporal: the contiguous range E_k of the schedule S, P:L78,
// P:L80), calls compare() (Alg. 1 l.14 P:L64) and atomically appends results
// to a fixed-size buffer (l.16 P:L66), re-invoking the kernel on overflow
// (P:L47).
//
// Here:
//   * queries are keyed and radix-sorted by the same (bin, cell) key as the
//     entries, so adjacent warps read the same cells (L1/L2 reuse) -- the
//     generalisation of "Q sorted by t_start";
//   * one warp per query: lanes probe the query's stencil of (bin, cell)
//     keys in parallel (bins filtered by their [min t_start, max t_end]
//     extent, the B_start/B_end test of P:L76), a warp scan flattens the runs
//     into one candidate sequence, and the 32 lanes stream 32 consecutive
//     candidates at a time with four 128-bit loads each (warp-cooperative
//     candidate tiles instead of one thread per query);
//   * refinement in fp64 (readings c1-c4, c8), rejecting on cheap tests before
//     any sqrt or divide;
//   * pass 1 counts per query, an exclusive scan gives exact offsets, pass 2
//     writes each result at offset + ballot rank (no result-buffer overflow,
//     no re-invocation, deterministic); a per-query sort by entry id makes
//     the order canonical (reading c7).
#include <algorithm>
#include <vector>

#include "internal.cuh"

namespace dts {
namespace {

constexpr int PT = 256;                 // threads per CTA in the pass kernels
constexpr int PW = PT / 32;             // warps per CTA (one query each)
constexpr int SMALL_SORT = 32;          // warp-register sort limit
constexpr int LARGE_SORT = 4096;        // CTA shared-memory sort limit

struct Counters {                       // device-side statistics / flags
    unsigned long long candidates;
    unsigned long long lookups;
    unsigned int max_count;
    unsigned int n_large;
    unsigned int bad;
    unsigned int pad;
};

// Query in the velocity form used by the refinement.
struct QState {
    double t0, t1;
    double x0, vx, y0, vy, z0, vz;
};

// ------------------------------------------------------------- refinement
// compare() of Alg. 1 l.14 for one (query, entry) pair, readings
// c1-c4: strict temporal overlap [ts, te]; relative position
// A(s) = A0 + s W, s = t - ts in [0, L]; |A(s)|^2 - d^2 = aa s^2 + 2 bb s + cc;
// the closed set where it is <= 0, intersected with [0, L].
__device__ __forceinline__ bool refine(const QState& q, const double2 st, const double2 sx,
                                       const double2 sy, const double2 sz, const double d2,
                                       double& t_out0, double& t_out1) {
    const double ts = fmax(q.t0, st.x);
    const double te = fmin(q.t1, st.y);
    if (!(ts < te)) return false;
    const double dq = ts - q.t0, de = ts - st.x;
    const double ax = fma(de, sx.y, sx.x) - fma(dq, q.vx, q.x0);
    const double ay = fma(de, sy.y, sy.x) - fma(dq, q.vy, q.y0);
    const double az = fma(de, sz.y, sz.x) - fma(dq, q.vz, q.z0);
    const double wx = sx.y - q.vx, wy = sy.y - q.vy, wz = sz.y - q.vz;
    const double cc = fma(ax, ax, fma(ay, ay, fma(az, az, -d2)));
    const double bb = fma(ax, wx, fma(ay, wy, az * wz));
    if (cc > 0.0 && bb >= 0.0) return false;          // outside and not approaching
    const double aa = fma(wx, wx, fma(wy, wy, wz * wz));
    const double L = te - ts;
    double lo, hi;
    if (aa == 0.0) {                                  // no relative motion
        if (!(cc <= 0.0)) return false;
        lo = 0.0;
        hi = L;
    } else {
        const double disc = fma(bb, bb, -aa * cc);
        if (disc < 0.0) return false;                 // never within d
        const double r = sqrt(disc);
        const double qq = -(bb + copysign(r, bb));
        double s1, s2;
        if (qq == 0.0) {
            s1 = s2 = -bb / aa;
        } else {
            const double x1 = qq / aa, x2 = cc / qq;
            s1 = fmin(x1, x2);
            s2 = fmax(x1, x2);
        }
        lo = fmax(s1, 0.0);
        hi = fmin(s2, L);
        if (lo > hi) return false;
    }
    t_out0 = ts + lo;
    t_out1 = hi >= L ? te : ts + hi;
    return true;
}

__device__ __forceinline__ bool load_query(const double4* __restrict__ Q, uint32_t qid, QState& q,
                                           double qlo[3], double qhi[3]) {
    const double4 s0 = Q[2 * (size_t)qid], s1 = Q[2 * (size_t)qid + 1];
    q.t0 = s0.x;
    q.t1 = s1.x;
    const double dur = s1.x - s0.x;
    const double p0[3] = {s0.y, s0.z, s0.w}, p1[3] = {s1.y, s1.z, s1.w};
    double v[3];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        v[a] = dur > 0.0 ? (p1[a] - p0[a]) / dur : 0.0;
        qlo[a] = fmin(p0[a], p1[a]);
        qhi[a] = fmax(p0[a], p1[a]);
    }
    q.x0 = p0[0]; q.vx = v[0];
    q.y0 = p0[1]; q.vy = v[1];
    q.z0 = p0[2]; q.vz = v[2];
    bool fin = isfinite(dur);
#pragma unroll
    for (int a = 0; a < 3; ++a) fin = fin && isfinite(p0[a]) && isfinite(p1[a]) && isfinite(v[a]);
    // a zero-duration query never overlaps strictly (c2); invalid queries are
    // reported by k_qkeys and must not drive the stencil loops
    return fin && dur > 0.0;
}

// --------------------------------------------------------------- query prep
__global__ void __launch_bounds__(PT) k_qkeys(const double4* __restrict__ Q, uint32_t nq,
                                             GridParams g, int have_grid,
                                             unsigned long long* __restrict__ keys,
                                             uint32_t* __restrict__ ids,
                                             Counters* __restrict__ ctr) {
    uint32_t i = blockIdx.x * PT + threadIdx.x;
    if (i >= nq) return;
    const double4 s0 = Q[2 * (size_t)i], s1 = Q[2 * (size_t)i + 1];
    const double c[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
    unsigned bad = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) if (!isfinite(c[k])) bad |= 1;
    if (!bad && s1.x < s0.x) bad |= 2;
    if (!bad) {
        const double dur = s1.x - s0.x;
#pragma unroll
        for (int a = 1; a < 4; ++a) {
            double e = fabs(c[4 + a] - c[a]);
            if (!isfinite(e) || (dur > 0.0 && !isfinite(e / dur))) bad |= 4;
        }
    }
    if (bad) atomicOr(&ctr->bad, bad);
    unsigned long long key = 0;
    if (have_grid && !bad)
        key = make_key(g, bin_of(g, s0.x), cell_of(g, 0, 0.5 * (s0.y + s1.y)),
                       cell_of(g, 1, 0.5 * (s0.z + s1.z)), cell_of(g, 2, 0.5 * (s0.w + s1.w)));
    keys[i] = key;
    ids[i] = i;
}

// ------------------------------------------------------- fused pass kernel
struct PassArgs {
    const double4* Q;
    const uint32_t* order;         // sorted position -> query id
    uint32_t nq;
    double d;
    GridParams g;
    SegSoA soa;
    HashTable ht;
    const double* bin_t0min;
    const double* bin_t1max;
    uint32_t* counts;              // per query id
    const unsigned long long* offsets;
    dts_result* out;
    uint32_t qid_base;
    uint32_t* large;               // query ids with count > SMALL_SORT
    Counters* ctr;
};

template <bool SCATTER>
__global__ void __launch_bounds__(PT) k_pass(const PassArgs a) {
    __shared__ uint32_t s_start[PW][32];
    __shared__ uint32_t s_excl[PW][32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t sq = blockIdx.x * PW + warp;
    if (sq >= a.nq) return;
    const uint32_t qid = a.order[sq];
    QState q;
    double qlo[3], qhi[3];
    const bool live = load_query(a.Q, qid, q, qlo, qhi);
    const GridParams& g = a.g;
    const double d = a.d, d2 = d * d;

    uint32_t my_hits = 0;
    unsigned long long out_pos = SCATTER ? a.offsets[qid] : 0ull;
    unsigned long long n_cand = 0, n_look = 0;

    if (live) {
        // temporal stencil: entries with t_start in (q.t0 - maxdur, q.t1)
        const double mt = 1e-12 * (fabs(q.t0) + g.maxdur);
        const int32_t lb = bin_of(g, q.t0 - g.maxdur - mt);
        const int32_t hb = bin_of(g, q.t1);
        // spatial stencil: MBB midpoint within d + half extent of the query MBB
        int32_t clo[3], cn[3];
#pragma unroll
        for (int ax = 0; ax < 3; ++ax) {
            const double ms = 1e-12 * (fabs(qlo[ax]) + fabs(qhi[ax]) + fabs(g.o[ax]) + d +
                                       g.half_ext[ax]);
            const double r = d + g.half_ext[ax] + ms;
            clo[ax] = cell_of(g, ax, qlo[ax] - r);
            cn[ax] = cell_of(g, ax, qhi[ax] + r) - clo[ax] + 1;
        }
        const unsigned long long ncomb = (unsigned long long)(hb - lb + 1) * (unsigned)cn[0] *
                                         (unsigned)cn[1] * (unsigned)cn[2];
        const unsigned long long nyx = (unsigned long long)cn[0] * (unsigned)cn[1];
        const unsigned long long nzyx = nyx * (unsigned)cn[2];
        for (unsigned long long c0 = 0; c0 < ncomb; c0 += 32) {
            // ---- lookups: one (bin, cell) per lane
            const unsigned long long c = c0 + lane;
            uint32_t start = 0, cnt = 0;
            if (c < ncomb) {
                const int32_t bin = lb + (int32_t)(c / nzyx);
                unsigned long long r = c % nzyx;
                const int32_t cz = clo[2] + (int32_t)(r / nyx);
                r %= nyx;
                const int32_t cy = clo[1] + (int32_t)(r / (unsigned)cn[0]);
                const int32_t cx = clo[0] + (int32_t)(r % (unsigned)cn[0]);
                if (__ldg(&a.bin_t0min[bin]) < q.t1 && __ldg(&a.bin_t1max[bin]) > q.t0) {
                    const unsigned long long key = make_key(g, bin, cx, cy, cz);
                    unsigned long long h = hash_key(key, a.ht.log2cap);
                    ++n_look;
                    while (true) {
                        const ulonglong2 sl =
                            __ldg(reinterpret_cast<const ulonglong2*>(a.ht.slots) + h);
                        if (sl.x == key) {
                            start = (uint32_t)sl.y;
                            cnt = (uint32_t)(sl.y >> 32) - start;
                            break;
                        }
                        if (sl.x == EMPTY_KEY) break;
                        h = (h + 1) & a.ht.mask;
                    }
                }
            }
            // ---- flatten the up-to-32 runs into one candidate sequence
            uint32_t incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += u;
            }
            const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
            __syncwarp();
            s_start[warp][lane] = start;
            s_excl[warp][lane] = incl - cnt;
            __syncwarp();
            n_cand += total;
            // ---- stream candidates 32 at a time
            for (uint32_t base = 0; base < total; base += 32) {
                const uint32_t t = base + lane;
                bool hit = false;
                double r0 = 0.0, r1 = 0.0;
                uint32_t p = 0;
                if (t < total) {
                    int j = 0;
#pragma unroll
                    for (int step = 16; step; step >>= 1)
                        if (s_excl[warp][j + step] <= t) j += step;
                    p = s_start[warp][j] + (t - s_excl[warp][j]);
                    const double2 st = __ldg(a.soa.st + p);
                    const double2 sx = __ldg(a.soa.sx + p);
                    const double2 sy = __ldg(a.soa.sy + p);
                    const double2 sz = __ldg(a.soa.sz + p);
                    hit = refine(q, st, sx, sy, sz, d2, r0, r1);
                }
                if (SCATTER) {
                    const uint32_t bal = __ballot_sync(0xffffffffu, hit);
                    if (hit) {
                        const unsigned long long pos =
                            out_pos + __popc(bal & ((1u << lane) - 1u));
                        dts_result rr;
                        rr.query_id = qid + a.qid_base;
                        rr.entry_id = __ldg(a.soa.eid + p);
                        rr.t_start = r0;
                        rr.t_end = r1;
                        a.out[pos] = rr;
                    }
                    out_pos += __popc(bal);
                } else {
                    my_hits += hit ? 1u : 0u;
                }
            }
        }
    }
    if (!SCATTER) {
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            my_hits += __shfl_xor_sync(0xffffffffu, my_hits, o);
            n_look += __shfl_xor_sync(0xffffffffu, n_look, o);
        }
        if (lane == 0) {
            a.counts[qid] = my_hits;
            atomicAdd(&a.ctr->candidates, n_cand);
            atomicAdd(&a.ctr->lookups, n_look);
            if (my_hits) atomicMax(&a.ctr->max_count, my_hits);
            if (my_hits > (uint32_t)SMALL_SORT) {
                uint32_t slot = atomicAdd(&a.ctr->n_large, 1u);
                a.large[slot] = qid;
            }
        }
    }
}

// ------------------------------------------------------ canonical order
// One warp per query with 2..32 results: bitonic sort by entry id across
// lanes (entry ids of one query are distinct), payload moved by shuffles.
__global__ void __launch_bounds__(PT) k_canon_small(const uint32_t* __restrict__ counts,
                                                   const unsigned long long* __restrict__ offsets,
                                                   uint32_t nq, const dts_result* __restrict__ raw,
                                                   dts_result* __restrict__ out) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t q = blockIdx.x * PW + warp;
    if (q >= nq) return;
    const uint32_t cnt = counts[q];
    if (cnt == 0 || cnt > (uint32_t)SMALL_SORT) return;
    const unsigned long long base = offsets[q];
    if (cnt == 1) {
        if (lane == 0) out[base] = raw[base];
        return;
    }
    uint32_t key = 0xffffffffu, qq = 0;
    double t0 = 0.0, t1 = 0.0;
    if ((uint32_t)lane < cnt) {
        const dts_result r = raw[base + lane];
        key = r.entry_id;
        qq = r.query_id;
        t0 = r.t_start;
        t1 = r.t_end;
    }
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const uint32_t ok = __shfl_xor_sync(0xffffffffu, key, j);
            const double o0 = __shfl_xor_sync(0xffffffffu, t0, j);
            const double o1 = __shfl_xor_sync(0xffffffffu, t1, j);
            const bool up = ((lane & k) == 0);
            const bool lower = ((lane & j) == 0);
            const bool take = lower == up ? (ok < key) : (ok > key);
            if (take) {
                key = ok;
                t0 = o0;
                t1 = o1;
            }
        }
    }
    qq = __shfl_sync(0xffffffffu, qq, 0);
    if ((uint32_t)lane < cnt) {
        dts_result r;
        r.query_id = qq;
        r.entry_id = key;
        r.t_start = t0;
        r.t_end = t1;
        out[base + lane] = r;
    }
}

// One CTA per query with 33..LARGE_SORT results: bitonic sort of
// (entry id << 32 | local index) in shared memory, then gather.
__global__ void __launch_bounds__(PT) k_canon_large(const uint32_t* __restrict__ large,
                                                   const Counters* __restrict__ ctr,
                                                   const uint32_t* __restrict__ counts,
                                                   const unsigned long long* __restrict__ offsets,
                                                   const dts_result* __restrict__ raw,
                                                   dts_result* __restrict__ out) {
    __shared__ unsigned long long sk[LARGE_SORT];
    const uint32_t nl = ctr->n_large;
    for (uint32_t i = blockIdx.x; i < nl; i += gridDim.x) {
        const uint32_t q = large[i];
        const uint32_t cnt = counts[q];
        if (cnt > (uint32_t)LARGE_SORT) continue;     // host path
        const unsigned long long base = offsets[q];
        uint32_t P = 64;
        while (P < cnt) P <<= 1;
        for (uint32_t j = threadIdx.x; j < P; j += PT)
            sk[j] = j < cnt ? ((unsigned long long)raw[base + j].entry_id << 32) | j : ~0ull;
        __syncthreads();
        for (uint32_t k = 2; k <= P; k <<= 1) {
            for (uint32_t jj = k >> 1; jj > 0; jj >>= 1) {
                for (uint32_t t = threadIdx.x; t < P; t += PT) {
                    const uint32_t u = t ^ jj;
                    if (u > t) {
                        const unsigned long long x = sk[t], y = sk[u];
                        const bool up = (t & k) == 0;
                        if ((x > y) == up) {
                            sk[t] = y;
                            sk[u] = x;
                        }
                    }
                }
                __syncthreads();
            }
        }
        for (uint32_t j = threadIdx.x; j < cnt; j += PT)
            out[base + j] = raw[base + (uint32_t)(sk[j] & 0xffffffffull)];
        __syncthreads();
    }
}

// Huge segments (> LARGE_SORT results of one query): radix sort by entry id.
__global__ void k_seg_keys(const dts_result* __restrict__ raw, uint32_t cnt,
                           unsigned long long* __restrict__ keys, uint32_t* __restrict__ idx) {
    uint32_t j = blockIdx.x * PT + threadIdx.x;
    if (j < cnt) {
        keys[j] = raw[j].entry_id;
        idx[j] = j;
    }
}
__global__ void k_seg_gather(const dts_result* __restrict__ raw, uint32_t cnt,
                             const uint32_t* __restrict__ idx, dts_result* __restrict__ out) {
    uint32_t j = blockIdx.x * PT + threadIdx.x;
    if (j < cnt) out[j] = raw[idx[j]];
}

__global__ void k_validate_only(const double4* __restrict__ Q, uint32_t nq, Counters* ctr) {
    uint32_t i = blockIdx.x * PT + threadIdx.x;
    if (i >= nq) return;
    const double4 s0 = Q[2 * (size_t)i], s1 = Q[2 * (size_t)i + 1];
    const double c[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
    unsigned bad = 0;
    for (int k = 0; k < 8; ++k) if (!isfinite(c[k])) bad |= 1;
    if (!bad && s1.x < s0.x) bad |= 2;
    if (bad) atomicOr(&ctr->bad, bad);
}

inline unsigned blocks(size_t n, int per) { return (unsigned)((n + per - 1) / per); }

struct EventTimer {
    bool on;
    cudaStream_t s;
    cudaEvent_t ev[6];
    int k = 0;
    EventTimer(bool enable, cudaStream_t st) : on(enable), s(st) {
        if (on) for (auto& e : ev) DTS_CUDA(cudaEventCreate(&e));
    }
    void mark() { if (on) DTS_CUDA(cudaEventRecord(ev[k++], s)); }
    float ms(int i) {
        float t = 0.f;
        if (on && i + 1 < k) cudaEventElapsedTime(&t, ev[i], ev[i + 1]);
        return t;
    }
    ~EventTimer() { if (on) for (auto& e : ev) cudaEventDestroy(e); }
};

}  // namespace

void search_device(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                   uint32_t qid_base, cudaStream_t s, SearchOut* out, dts_search_stats* stats) {
    out->results = nullptr;
    out->count = 0;
    dts_search_stats local{};
    if (stats) local.time_kernels = stats->time_kernels;
    if (nq == 0) {
        if (stats) *stats = local;
        return;
    }
    const double4* Q = reinterpret_cast<const double4*>(Q_dev);
    DevBuf<Counters> ctr(1, s);
    DTS_CUDA(cudaMemsetAsync(ctr.p, 0, sizeof(Counters), s));

    if (idx->n == 0) {   // empty index: validate only
        k_validate_only<<<blocks(nq, PT), PT, 0, s>>>(Q, (uint32_t)nq, ctr.p);
        DTS_LAUNCH_CHECK();
        Counters hc;
        DTS_CUDA(cudaMemcpyAsync(&hc, ctr.p, sizeof(hc), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        if (hc.bad) throw Error(DTS_EINVAL, "invalid query segment (non-finite or t_end < t_start)");
        if (stats) *stats = local;
        return;
    }

    EventTimer tm(local.time_kernels != 0, s);
    tm.mark();
    // ---- query prep: key + sort
    DevBuf<unsigned long long> qk(nq, s), qk_tmp(nq, s);
    DevBuf<uint32_t> order(nq, s), order_tmp(nq, s);
    k_qkeys<<<blocks(nq, PT), PT, 0, s>>>(Q, (uint32_t)nq, idx->gp, 1, qk.p, order.p, ctr.p);
    DTS_LAUNCH_CHECK();
    radix_sort_pairs(qk.p, order.p, qk_tmp.p, order_tmp.p, nq, idx->key_bits, s);
    qk_tmp.release();
    order_tmp.release();
    qk.release();
    tm.mark();

    // ---- pass 1: count
    DevBuf<uint32_t> counts(nq, s), large(nq, s);
    DevBuf<unsigned long long> offsets(nq + 1, s);
    PassArgs pa;
    pa.Q = Q;
    pa.order = order.p;
    pa.nq = (uint32_t)nq;
    pa.d = d;
    pa.g = idx->gp;
    pa.soa = idx->soa;
    pa.ht = idx->ht;
    pa.bin_t0min = idx->bin_t0min;
    pa.bin_t1max = idx->bin_t1max;
    pa.counts = counts.p;
    pa.offsets = offsets.p;
    pa.out = nullptr;
    pa.qid_base = qid_base;
    pa.large = large.p;
    pa.ctr = ctr.p;
    k_pass<false><<<blocks(nq, PW), PT, 0, s>>>(pa);
    DTS_LAUNCH_CHECK();
    tm.mark();
    scan_exclusive_u32_to_u64(counts.p, offsets.p, nq, s);
    tm.mark();

    struct {
        Counters c;
        unsigned long long total;
    } h;
    DTS_CUDA(cudaMemcpyAsync(&h.c, ctr.p, sizeof(Counters), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaMemcpyAsync(&h.total, offsets.p + nq, sizeof(unsigned long long),
                             cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    if (h.c.bad & 1) throw Error(DTS_EINVAL, "query segment with a non-finite coordinate or time");
    if (h.c.bad & 2) throw Error(DTS_EINVAL, "query segment with t_end < t_start");
    if (h.c.bad & 4) throw Error(DTS_EINVAL, "query segment whose speed overflows fp64");
    local.candidates = h.c.candidates;
    local.cell_lookups = h.c.lookups;
    local.results = h.total;
    local.max_results_per_query = h.c.max_count;

    if (h.total > 0) {
        // ---- pass 2: scatter at exact offsets, then canonical order
        DevBuf<dts_result> raw(h.total, s);
        dts_result* fin = nullptr;
        DTS_CUDA(cudaMallocAsync((void**)&fin, h.total * sizeof(dts_result), s));
        try {
            pa.out = raw.p;
            k_pass<true><<<blocks(nq, PW), PT, 0, s>>>(pa);
            DTS_LAUNCH_CHECK();
            tm.mark();
            k_canon_small<<<blocks(nq, PW), PT, 0, s>>>(counts.p, offsets.p, (uint32_t)nq, raw.p,
                                                        fin);
            DTS_LAUNCH_CHECK();
            if (h.c.n_large) {
                const unsigned g = (unsigned)std::min<uint32_t>(h.c.n_large, 148 * 4);
                k_canon_large<<<g, PT, 0, s>>>(large.p, ctr.p, counts.p, offsets.p, raw.p, fin);
                DTS_LAUNCH_CHECK();
            }
            if (h.c.max_count > (uint32_t)LARGE_SORT) {
                std::vector<uint32_t> hl(h.c.n_large);
                DTS_CUDA(cudaMemcpyAsync(hl.data(), large.p, hl.size() * sizeof(uint32_t),
                                         cudaMemcpyDeviceToHost, s));
                DTS_CUDA(cudaStreamSynchronize(s));
                for (uint32_t qh : hl) {
                    uint32_t cnt;
                    unsigned long long base;
                    DTS_CUDA(cudaMemcpyAsync(&cnt, counts.p + qh, 4, cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaMemcpyAsync(&base, offsets.p + qh, 8, cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                    if (cnt <= (uint32_t)LARGE_SORT) continue;
                    DevBuf<unsigned long long> k1(cnt, s), k2(cnt, s);
                    DevBuf<uint32_t> v1(cnt, s), v2(cnt, s);
                    k_seg_keys<<<blocks(cnt, PT), PT, 0, s>>>(raw.p + base, cnt, k1.p, v1.p);
                    DTS_LAUNCH_CHECK();
                    radix_sort_pairs(k1.p, v1.p, k2.p, v2.p, cnt,
                                     bits_for(idx->n ? idx->n - 1 : 0), s);
                    k_seg_gather<<<blocks(cnt, PT), PT, 0, s>>>(raw.p + base, cnt, v1.p,
                                                                fin + base);
                    DTS_LAUNCH_CHECK();
                }
            }
            tm.mark();
            DTS_CUDA(cudaStreamSynchronize(s));
        } catch (...) {
            cudaFreeAsync(fin, s);
            throw;
        }
        out->results = fin;
        out->count = (size_t)h.total;
    } else {
        tm.mark();
        tm.mark();
    }
    if (local.time_kernels) {
        DTS_CUDA(cudaStreamSynchronize(s));
        local.ms_prep = tm.ms(0);
        local.ms_count = tm.ms(1);
        local.ms_scan = tm.ms(2);
        local.ms_scatter = tm.ms(3);
        local.ms_canon = tm.ms(4);
    }
    if (stats) *stats = local;
}

}  // namespace dts
