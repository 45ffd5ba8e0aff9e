// build.cu -- GPU index builder.
//
// The paper builds its indexes on the host (P:L76 temporal bins over D sorted
// by t_start; P:L44 flatly structured grid of non-empty cells G with a lookup
// array A; P:L86-P:L87 spatial subbins sized by the max per-dimension extent).
// Here the index is built on the device and each entry is stored once:
//
//   1. k_bounds       fp64 min/max reduction: t_min, t_max, spatial
//                     bounds and max per-axis extent (P:L86-P:L87), max
//                     duration; validation of every segment.
//   2. host           bin width b, cell widths w_a >= extent_a + d_hint.
//   3. k_keys         key = (bin of t_start, cell of the MBB midpoint), row-major
//                     (bin, z, y, x) so that x-adjacent cells are adjacent runs.
//   4. radix sort     stable (key, id): within a cell entries stay in id order.
//   5. k_gather_cells sorted SoA double2 streams (t0,t1) (x0,vx) (y0,vy) (z0,vz),
//                     fused with: bin offsets (B_first of P:L76), per-bin
//                     [min t_start, max t_end] extents (B_start/B_end of
//                     P:L76) with CTA-aggregated atomics, non-empty cell count.
//   6. k_insert       non-empty cells ->
//                     open-addressing hash table key -> [start, end) (the role
//                     of G and A of P:L44, with no duplicated ids since every
//                     entry is in exactly one cell).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "internal.cuh"

namespace dts {
namespace {

struct Bounds {
    double tmin, tmax;
    double lo[3], hi[3];
    double ext[3];             // max extent per axis (outliers excluded when thresholds apply)
    double maxdur;             // max duration (idem)
    double absmax;
    double sext[3], sdur;      // sums of extents and durations (sample means)
    unsigned long long cnt;    // valid entries added
    unsigned long long nout;   // outliers (extent or duration above the thresholds)
    int bad;
};

// Outlier thresholds (build.cu header of internal.cuh "outliers"): an entry
// whose extent exceeds ext[a] on some axis or whose duration exceeds dur.
struct Thresh {
    double ext[3], dur;
    int on;
};

constexpr int BT = 256;

__device__ __forceinline__ void bounds_init(Bounds& b) {
    b.tmin = INFINITY; b.tmax = -INFINITY;
    for (int a = 0; a < 3; ++a) {
        b.lo[a] = INFINITY; b.hi[a] = -INFINITY; b.ext[a] = 0.0; b.sext[a] = 0.0;
    }
    b.maxdur = 0.0; b.absmax = 0.0; b.sdur = 0.0; b.cnt = 0; b.nout = 0; b.bad = 0;
}

__device__ __forceinline__ void bounds_merge(Bounds& b, const Bounds& o) {
    b.tmin = fmin(b.tmin, o.tmin); b.tmax = fmax(b.tmax, o.tmax);
    for (int a = 0; a < 3; ++a) {
        b.lo[a] = fmin(b.lo[a], o.lo[a]); b.hi[a] = fmax(b.hi[a], o.hi[a]);
        b.ext[a] = fmax(b.ext[a], o.ext[a]);
    }
    b.maxdur = fmax(b.maxdur, o.maxdur); b.absmax = fmax(b.absmax, o.absmax);
    for (int a = 0; a < 3; ++a) b.sext[a] += o.sext[a];
    b.sdur += o.sdur; b.cnt += o.cnt; b.nout += o.nout;
    b.bad |= o.bad;
}

// Field by field (shuffle, then merge): no second Bounds held in registers.
__device__ __forceinline__ void bounds_shfl(Bounds& b, int off) {
    const unsigned F = 0xffffffffu;
    b.tmin = fmin(b.tmin, __shfl_xor_sync(F, b.tmin, off));
    b.tmax = fmax(b.tmax, __shfl_xor_sync(F, b.tmax, off));
    for (int a = 0; a < 3; ++a) {
        b.lo[a] = fmin(b.lo[a], __shfl_xor_sync(F, b.lo[a], off));
        b.hi[a] = fmax(b.hi[a], __shfl_xor_sync(F, b.hi[a], off));
        b.ext[a] = fmax(b.ext[a], __shfl_xor_sync(F, b.ext[a], off));
        b.sext[a] += __shfl_xor_sync(F, b.sext[a], off);
    }
    b.maxdur = fmax(b.maxdur, __shfl_xor_sync(F, b.maxdur, off));
    b.absmax = fmax(b.absmax, __shfl_xor_sync(F, b.absmax, off));
    b.sdur += __shfl_xor_sync(F, b.sdur, off);
    b.cnt += __shfl_xor_sync(F, b.cnt, off);
    b.nout += __shfl_xor_sync(F, b.nout, off);
    b.bad |= __shfl_xor_sync(F, b.bad, off);
}

__device__ void block_reduce_write(Bounds& b, Bounds* out) {
    __shared__ Bounds sm[BT / 32];
    for (int off = 16; off; off >>= 1) bounds_shfl(b, off);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (lane == 0) sm[warp] = b;
    __syncthreads();
    if (warp == 0) {
        Bounds c;
        if (lane < BT / 32) c = sm[lane]; else bounds_init(c);
        for (int off = 16; off; off >>= 1) bounds_shfl(c, off);
        if (lane == 0) *out = c;
    }
}

// Segment validity (readings c4, c8): finite coordinates and times,
// t_end >= t_start, finite velocity.  With thresholds, an outlier counts in
// the time range but not in the spatial bounds, the max extent and the
// duration that size the grid and the stencils; returns whether the entry
// is an outlier.
__device__ __forceinline__ bool is_outlier(const Thresh& th, const double4 s0, const double4 s1) {
    return th.on && (fabs(s1.y - s0.y) > th.ext[0] || fabs(s1.z - s0.z) > th.ext[1] ||
                     fabs(s1.w - s0.w) > th.ext[2] || s1.x - s0.x > th.dur);
}

template <bool SUMS = true>
__device__ __forceinline__ bool bounds_add(Bounds& b, const double4 s0, const double4 s1,
                                           const Thresh& th) {
    // (t0,x0,y0,z0), (t1,x1,y1,z1); v - v is 0 for a finite v and NaN
    // otherwise, so one comparison checks all eight values
    const double z = ((s0.x - s0.x) + (s1.x - s1.x)) + ((s0.y - s0.y) + (s1.y - s1.y)) +
                     ((s0.z - s0.z) + (s1.z - s1.z)) + ((s0.w - s0.w) + (s1.w - s1.w));
    if (!(z == 0.0)) { b.bad |= 1; return false; }
    if (s1.x < s0.x) { b.bad |= 2; return false; }
    const bool outl = is_outlier(th, s0, s1);
    const double dur = s1.x - s0.x;
    b.tmin = fmin(b.tmin, s0.x);
    b.tmax = fmax(b.tmax, s1.x);
    if (!outl) b.maxdur = fmax(b.maxdur, dur);
    if (SUMS) {
        b.sdur += dur;
        b.cnt += 1;
    }
    b.nout += outl ? 1ull : 0ull;
    const double p0[3] = {s0.y, s0.z, s0.w}, p1[3] = {s1.y, s1.z, s1.w};
    double emax = 0.0;
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        const double lo = fmin(p0[a], p1[a]), hi = fmax(p0[a], p1[a]);
        const double e = hi - lo;
        if (SUMS) b.sext[a] += e;
        if (!outl) {
            // the grid's domain is the main entries' (an outlier's copies
            // clamp into the boundary cells like any point outside it)
            b.lo[a] = fmin(b.lo[a], lo);
            b.hi[a] = fmax(b.hi[a], hi);
            b.ext[a] = fmax(b.ext[a], e);
        }
        emax = fmax(emax, e);
    }
    // speed |p1 - p0| / dur must be finite on every axis: an infinite extent,
    // or (only possible for dur < 1) an overflowing quotient of the largest
    // extent (division is monotone in the numerator)
    if (!isfinite(emax) || (dur > 0.0 && dur < 1.0 && !isfinite(emax / dur))) b.bad |= 4;
    return outl;
}

__global__ void __launch_bounds__(BT) k_bounds(const double4* __restrict__ D, size_t n,
                                              Bounds* __restrict__ partial) {
    Bounds b;
    bounds_init(b);
    for (size_t i = (size_t)blockIdx.x * BT + threadIdx.x; i < n; i += (size_t)gridDim.x * BT)
        bounds_add(b, ld256(D + 2 * i), ld256(D + 2 * i + 1), Thresh{{0, 0, 0}, 0, 0});
    block_reduce_write(b, &partial[blockIdx.x]);
}

// Bounds of the S entries i = floor(j n / S), j < S: the provisional grid of
// the fused bounds + keys pass (any grid gives the same results -- the
// stencils use the exact extents; see build_index_device).  A periodic input
// can alias with the stride (trajectory-major D with a stride that is a
// multiple of the segments per trajectory samples one time step): the build
// then finds the exact time range well outside the sampled one and redoes
// the keys with the exact grid.  (Hashed offsets inside each stride
// avoid the aliasing but measured 2.5% slower on C4: the grid they give
// hashes the 8-cell blocks less evenly -- a Fibonacci hash spreads the
// arithmetic progressions of the old grid's block keys better than random.)
__global__ void __launch_bounds__(BT) k_bounds_sample(const double4* __restrict__ D, size_t n,
                                                     size_t S, Bounds* __restrict__ partial,
                                                     const Thresh* __restrict__ thp) {
    const Thresh th = thp ? *thp : Thresh{{0, 0, 0}, 0, 0};
    Bounds b;
    bounds_init(b);
    for (size_t j = (size_t)blockIdx.x * BT + threadIdx.x; j < S; j += (size_t)gridDim.x * BT) {
        const size_t i = (size_t)(((unsigned __int128)j * n) / S);
        bounds_add(b, D[2 * i], D[2 * i + 1], th);
    }
    block_reduce_write(b, &partial[blockIdx.x]);
}

// Outlier thresholds from the sample's bounds (grid method): 8x the mean
// extent per axis and the mean duration, at least a thousandth of the
// sample's span (on the device: the second sample pass follows without a
// host round trip).
struct SampleOut {
    Bounds b;          // the sample's bounds without the outliers
    Thresh th;
};
__global__ void k_thresh(const Bounds* __restrict__ b, Thresh* __restrict__ th) {
    const Bounds x = *b;
    Thresh t{{0, 0, 0}, 0, 0};
    if (x.cnt > 0 && !x.bad) {
        const double c = (double)x.cnt;
        for (int a = 0; a < 3; ++a) t.ext[a] = fmax(8.0 * x.sext[a] / c, 1e-3 * (x.hi[a] - x.lo[a]));
        t.dur = fmax(8.0 * x.sdur / c, 1e-3 * (x.tmax - x.tmin));
        t.on = 1;
    }
    *th = t;
}

__global__ void __launch_bounds__(BT) k_bounds_final(const Bounds* __restrict__ partial, int np,
                                                    Bounds* __restrict__ out) {
    Bounds b;
    bounds_init(b);
    for (int i = threadIdx.x; i < np; i += BT) bounds_merge(b, partial[i]);
    // max |coordinate or time| of the valid entries = max |bound| (the
    // per-entry values need not be visited)
    if (b.tmin <= b.tmax) {
        b.absmax = fmax(fabs(b.tmin), fabs(b.tmax));
        for (int a = 0; a < 3; ++a) b.absmax = fmax(b.absmax, fmax(fabs(b.lo[a]), fabs(b.hi[a])));
    }
    block_reduce_write(b, out);
}

// Occupancy of the sample's bounding box: the midpoints of the S strided
// sample rows marked in a 32^3 bitmap over [lo, hi] (bounds read from the
// device).  The fraction of marked cells estimates how much of the box the
// data fills (C4's galaxy: 5%; C3's random walks: 60%).
constexpr int OCC_RES = 32;
__global__ void __launch_bounds__(BT) k_sample_occupancy(const double4* __restrict__ D, size_t n,
                                                        size_t S, const Bounds* __restrict__ bnd,
                                                        uint32_t* __restrict__ bitmap) {
    const Bounds b = *bnd;
    for (size_t j = (size_t)blockIdx.x * BT + threadIdx.x; j < S; j += (size_t)gridDim.x * BT) {
        const size_t i = (size_t)(((unsigned __int128)j * n) / S);
        const double4 s0 = D[2 * i], s1 = D[2 * i + 1];
        const double mid[3] = {0.5 * (s0.y + s1.y), 0.5 * (s0.z + s1.z), 0.5 * (s0.w + s1.w)};
        uint32_t cell = 0;
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const double span = b.hi[a] - b.lo[a];
            double f = span > 0.0 ? (mid[a] - b.lo[a]) / span * OCC_RES : 0.0;
            int c = (f > 0.0) ? (int)fmin(f, (double)(OCC_RES - 1)) : 0;
            cell = cell * OCC_RES + (uint32_t)c;
        }
        atomicOr(&bitmap[cell >> 5], 1u << (cell & 31u));
    }
}

// Sorted (key, row) pairs, either packed -- a[p] = key << shift | row, when
// key bits + row bits fit in 64 (a keys-only sort on the key bits then moves
// 8 bytes per element instead of 12) -- or as separate arrays (ids != null).
struct SortedKeys {
    const unsigned long long* a;
    int shift;
    const uint32_t* ids;
    __device__ __forceinline__ unsigned long long key(size_t p) const { return a[p] >> shift; }
    __device__ __forceinline__ uint32_t row(size_t p) const {
        return ids ? ids[p] : (uint32_t)(a[p] & ((1ull << shift) - 1ull));
    }
};

__global__ void __launch_bounds__(BT) k_keys(const double4* __restrict__ D, size_t n, GridParams g,
                                            unsigned long long* __restrict__ keys,
                                            uint32_t* __restrict__ ids, int shift) {
    size_t i = (size_t)blockIdx.x * BT + threadIdx.x;
    if (i >= n) return;
    double4 s0 = D[2 * i], s1 = D[2 * i + 1];
    int32_t bin = bin_of(g, s0.x);
    int32_t cx = cell_of(g, 0, 0.5 * (s0.y + s1.y));
    int32_t cy = cell_of(g, 1, 0.5 * (s0.z + s1.z));
    int32_t cz = cell_of(g, 2, 0.5 * (s0.w + s1.w));
    const unsigned long long k = make_key(g, bin, cx, cy, cz);
    if (ids) {
        keys[i] = k;
        ids[i] = (uint32_t)i;
    } else {
        keys[i] = (k << shift) | (unsigned long long)i;
    }
}

// One read of D for three things: the exact bounds and validation (as
// k_bounds), the packed sort keys under the provisional grid g (as k_keys),
// and the digit counts of every pass of the coming radix sort (as
// k_rs_hist_all) -- the separate kernels read D twice and the keys once more.

__device__ __forceinline__ unsigned long long packed_key(const GridParams& g, const double4 s0,
                                                         const double4 s1, int shift, size_t i) {
    const int32_t bin = bin_of(g, s0.x);
    const int32_t cx = cell_of(g, 0, 0.5 * (s0.y + s1.y));
    const int32_t cy = cell_of(g, 1, 0.5 * (s0.z + s1.z));
    const int32_t cz = cell_of(g, 2, 0.5 * (s0.w + s1.w));
    return (make_key(g, bin, cx, cy, cz) << shift) | (unsigned long long)i;
}

// Outliers (thresholds th): bit of the row in orows, row appended to olist
// (capacity ocap; ocount may exceed it: the build then drops outlier filing).
struct OutlierOut {
    uint32_t* orows;
    uint32_t* olist;
    unsigned int* ocount;
    unsigned int ocap;
};

__device__ __forceinline__ void note_outlier(const OutlierOut& oo, size_t i) {
    atomicOr(&oo.orows[i >> 5], 1u << (i & 31));
    const unsigned int k = atomicAdd(oo.ocount, 1u);
    if (k < oo.ocap) oo.olist[k] = (uint32_t)i;
}

// OUT: thresholds on (outliers flagged and listed); two entries in flight
// per thread step either way (one at a time with outliers measured 0.416 ms
// on C4 against 0.32 without)
template <int MINB, bool OUT>
__global__ void __launch_bounds__(BT, MINB) k_bounds_keys(const double4* __restrict__ D, size_t n,
                                                      GridParams g,
                                                      unsigned long long* __restrict__ keys,
                                                      int shift, const PassPlan plan,
                                                      Bounds* __restrict__ partial,
                                                      uint32_t* __restrict__ hist, Thresh th,
                                                      OutlierOut oo) {
    __shared__ uint32_t h[OS_MAXPASS * OS_HSTRIDE];
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += BT) h[j] = 0;
    __syncthreads();
    Bounds b;
    bounds_init(b);
    auto count = [&](unsigned long long v) {    // unrolled: the plan stays in registers
#pragma unroll
        for (int p = 0; p < OS_MAXPASS; ++p)
            if (p < plan.npass)
                atomicAdd(&h[p * OS_HSTRIDE + ((v >> plan.shift[p]) & ((1u << plan.bits[p]) - 1u))], 1u);
    };
    const size_t stride = (size_t)gridDim.x * BT;
    size_t i = (size_t)blockIdx.x * BT + threadIdx.x;
    const Thresh thr = OUT ? th : Thresh{{0, 0, 0}, 0, 0};
    for (; i + stride < n; i += 2 * stride) {      // two entries in flight per thread
        const size_t j = i + stride;
        const double4 a0 = ld256(D + 2 * i), a1 = ld256(D + 2 * i + 1);
        const double4 c0 = ld256(D + 2 * j), c1 = ld256(D + 2 * j + 1);
        const bool oa = bounds_add<false>(b, a0, a1, thr);
        const bool oc = bounds_add<false>(b, c0, c1, thr);
        const unsigned long long va = packed_key(g, a0, a1, shift, i);
        const unsigned long long vc = packed_key(g, c0, c1, shift, j);
        keys[i] = va;
        keys[j] = vc;
        count(va);
        count(vc);
        if (OUT && oa) note_outlier(oo, i);
        if (OUT && oc) note_outlier(oo, j);
    }
    if (i < n) {
        const double4 a0 = ld256(D + 2 * i), a1 = ld256(D + 2 * i + 1);
        const bool oa = bounds_add<false>(b, a0, a1, thr);
        const unsigned long long va = packed_key(g, a0, a1, shift, i);
        keys[i] = va;
        count(va);
        if (OUT && oa) note_outlier(oo, i);
    }
    block_reduce_write(b, &partial[blockIdx.x]);
    __syncthreads();
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += BT)
        if (h[j]) atomicAdd(hist + j, h[j]);
}

// The record of row i of D as the search sees it (velocity form, the same
// arithmetic as the gather).
__device__ __forceinline__ double velocity(double p0, double p1, double dur) {
    return dur > 0.0 ? (p1 - p0) / dur : 0.0;
}
__device__ __forceinline__ ORec orec_of(const double4* __restrict__ D, size_t i) {
    const double4 s0 = D[2 * i], s1 = D[2 * i + 1];
    const double dur = s1.x - s0.x;
    ORec o;
    o.t0 = s0.x;
    o.t1 = s1.x;
    o.x[0] = s0.y; o.x[1] = s0.z; o.x[2] = s0.w;
    o.v[0] = velocity(s0.y, s1.y, dur);
    o.v[1] = velocity(s0.z, s1.z, dur);
    o.v[2] = velocity(s0.w, s1.w, dur);
    return o;
}

// Copies of each listed outlier (cells of its sub-slice boxes, every bin of
// its time span); counts[i] saturates at OUT_MAX (the build then drops
// outlier filing).
constexpr unsigned int OUT_MAX = 1u << 20;
__global__ void __launch_bounds__(BT) k_outlier_count(const double4* __restrict__ D,
                                                     const uint32_t* __restrict__ olist,
                                                     uint32_t nout, GridParams g,
                                                     uint32_t* __restrict__ counts) {
    const uint32_t i = blockIdx.x * BT + threadIdx.x;
    if (i >= nout) return;
    const ORec o = orec_of(D, olist[i]);
    const int32_t jo0 = bin_of(g, o.t0), jo1 = bin_of(g, o.t1);
    unsigned long long c = 0;
    for (int32_t j = jo0; j <= jo1 && c < OUT_MAX; ++j)
        outlier_boxes(g, o, j, jo0, jo1, [&](const int32_t lo[3], const int32_t hi[3]) {
            c += (unsigned long long)(hi[0] - lo[0] + 1) * (unsigned long long)(hi[1] - lo[1] + 1) *
                 (unsigned long long)(hi[2] - lo[2] + 1);
        });
    counts[i] = (uint32_t)min(c, (unsigned long long)OUT_MAX);
}

// Packed keys (cell key << shift | row) of the copies at keys[off[i] ..],
// with their digit counts added to the sort's histograms.
__global__ void __launch_bounds__(BT) k_outlier_emit(const double4* __restrict__ D,
                                                    const uint32_t* __restrict__ olist,
                                                    uint32_t nout, GridParams g,
                                                    const unsigned long long* __restrict__ off,
                                                    unsigned long long* __restrict__ keys, int shift,
                                                    const PassPlan plan,
                                                    uint32_t* __restrict__ hist) {
    __shared__ uint32_t h[OS_MAXPASS * OS_HSTRIDE];
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += BT) h[j] = 0;
    __syncthreads();
    const uint32_t i = blockIdx.x * BT + threadIdx.x;
    if (i < nout) {
        const uint32_t row = olist[i];
        const ORec o = orec_of(D, row);
        const int32_t jo0 = bin_of(g, o.t0), jo1 = bin_of(g, o.t1);
        unsigned long long k = off[i];
        for (int32_t j = jo0; j <= jo1; ++j)
            outlier_boxes(g, o, j, jo0, jo1, [&](const int32_t lo[3], const int32_t hi[3]) {
                for (int32_t cz = lo[2]; cz <= hi[2]; ++cz)
                    for (int32_t cy = lo[1]; cy <= hi[1]; ++cy)
                        for (int32_t cx = lo[0]; cx <= hi[0]; ++cx) {
                            const unsigned long long v =
                                (make_key(g, j, cx, cy, cz) << shift) | (unsigned long long)row;
                            keys[k++] = v;
                            for (int p = 0; p < plan.npass; ++p)
                                atomicAdd(&h[p * OS_HSTRIDE +
                                             ((v >> plan.shift[p]) & ((1u << plan.bits[p]) - 1u))], 1u);
                        }
            });
    }
    __syncthreads();
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += BT)
        if (h[j]) atomicAdd(hist + j, h[j]);
}

// Block slots: the head of each block of 8 keys (the first sorted
// entry with that key >> 3) walks the block's entries -- keys ascend, so the
// offsets key & 7 come in order -- builds the 8 inclusive prefix counts and
// claims one 32-byte slot.  One CAS per block instead of one per cell.
__device__ __forceinline__ void insert_block(const HashTable& ht, unsigned long long blk,
                                             uint32_t start, uint32_t big,
                                             unsigned long long c_lo, unsigned long long c_hi) {
    unsigned long long b = bucket_of(blk, ht);
    BlockSlot* const slots = ht.blocks();
    while (true) {
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            BlockSlot& sl = slots[2 * b + i];
            if (atomicCAS(&sl.key, EMPTY_KEY, blk) == EMPTY_KEY) {
                // the rest of the slot in two stores: (start, big), cum[0..7]
                *reinterpret_cast<unsigned long long*>(&sl.start) =
                    (unsigned long long)start | ((unsigned long long)big << 32);
                *reinterpret_cast<ulonglong2*>(sl.cum) = make_ulonglong2(c_lo, c_hi);
                return;
            }
        }
        b = next_bucket(b, ht);
    }
}

// Block slots, lane-parallel: every block head walks its own block in the
// staged keys (blocks average ~4 entries on C4), counting the 8 key offsets
// as bytes of one u64 (c += 1 << 8 * (key & 7)); one multiply by
// 0x0101010101010101 then gives the 8 inclusive prefix counts.  A block
// longer than WALK entries is queued and done by a whole warp with ballots
// (as k_insert_blocks), so no lane walks a long block alone.
template <int ITEMS, int WALK>
__global__ void __launch_bounds__(BT) k_insert_blocks_lane(const SortedKeys keys, size_t n,
                                                          HashTable ht) {
    static_assert(WALK < 256, "byte counters");
    constexpr int TILE = BT * ITEMS;
    __shared__ unsigned long long s_key[TILE + 1];
    __shared__ uint32_t s_long[TILE];
    __shared__ uint32_t s_nlong;
    const size_t p0 = (size_t)blockIdx.x * TILE;
    const uint32_t tn = (uint32_t)min((size_t)TILE, n - p0);
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const uint32_t loc = k * BT + threadIdx.x;
        if (loc < tn) s_key[1 + loc] = keys.key(p0 + loc);
    }
    if (threadIdx.x == 0) {
        s_key[0] = p0 > 0 ? keys.key(p0 - 1) : ~0ull;
        s_nlong = 0;
    }
    __syncthreads();
    auto key_at = [&](uint32_t q) -> unsigned long long {   // tile position q (may be >= tn)
        if (q < tn) return s_key[1 + q];
        const size_t p = p0 + q;
        return p < n ? keys.key(p) : ~0ull;
    };
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const uint32_t loc = k * BT + threadIdx.x;
        if (loc >= tn) continue;
        const unsigned long long blk = s_key[1 + loc] >> 3;
        if (p0 + loc != 0 && (s_key[loc] >> 3) == blk) continue;
        unsigned long long c = 0;
        uint32_t q = loc;
        int steps = 0;
        unsigned long long kq = s_key[1 + loc];
        do {
            c += 1ull << (8 * (uint32_t)(kq & 7ull));
            ++q;
            ++steps;
            kq = key_at(q);
        } while ((kq >> 3) == blk && steps < WALK);
        if ((kq >> 3) == blk) {                 // longer than WALK: warp path below
            s_long[atomicAdd(&s_nlong, 1u)] = loc;
            continue;
        }
        const unsigned long long pre = c * 0x0101010101010101ull;   // byte j = cum[j]
        unsigned long long lo = 0, hi = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            lo |= ((pre >> (8 * j)) & 0xFFull) << (16 * j);
            hi |= ((pre >> (8 * (4 + j))) & 0xFFull) << (16 * j);
        }
        insert_block(ht, blk, (uint32_t)(p0 + loc), 0u, lo, hi);
    }
    __syncthreads();
    const uint32_t nl = s_nlong;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (uint32_t w = warp; w < nl; w += BT / 32) {
        const uint32_t hp = s_long[w];
        const unsigned long long hb = s_key[1 + hp] >> 3;
        uint32_t cum[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (uint32_t q = hp;; q += 32) {
            const unsigned long long kq = key_at(q + lane);
            const bool in = (kq >> 3) == hb;
            const uint32_t off = (uint32_t)(kq & 7ull);
#pragma unroll
            for (int j = 0; j < 8; ++j) cum[j] += __popc(__ballot_sync(0xffffffffu, in && off <= (uint32_t)j));
            if (__ballot_sync(0xffffffffu, in) != 0xffffffffu) break;
        }
        if (lane == 0) {
            unsigned long long lo = 0, hi = 0;
            uint32_t big = 0;
            if (cum[7] > 65535u) {
                big = 1;
                lo = cum[7];
            } else {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    lo |= (unsigned long long)cum[j] << (16 * j);
                    hi |= (unsigned long long)cum[4 + j] << (16 * j);
                }
            }
            insert_block(ht, hb, (uint32_t)(p0 + hp), big, lo, hi);
        }
    }
}

// Block slots without walks: thread t owns the tile positions [t*ITEMS,
// (t+1)*ITEMS); a CTA-wide max-scan of the head positions gives every
// position the head of its block, and every position adds 1 to its block's
// counter of its key offset (16-bit lanes of two u64 per head, shared-memory
// atomics).  Heads then read their 8 counts, form the prefix counts with one
// multiply per half and claim a slot.  Only the tile's last block may
// continue past the tile: its head walks the global keys beyond (positions
// before the tile's first head belong to the previous tile's last block and
// are counted by that walk).
// Sorted position p <- original row ids[p]: ITEMS positions per thread
// (strided by the CTA so stores stay coalesced), all row loads issued first;
// the velocity form of each segment is written to the SoA streams.  Fused
// with the per-cell / per-bin bookkeeping of the sorted order (the tile's
// keys and bins are staged in shared memory with a one-element halo):
//   * non-empty cells are counted (key change between p - 1 and p);
//   * bin_start[0..m] (the entries of bin j are the sorted positions
//     [bin_start[j], bin_start[j+1]): the index range [B_first, B_last] of
//     P:L76, keys being bin-major);
//   * per-bin extents [min t_start, max t_end] (B_start / B_end of P:L76) with
//     one atomic pair per CTA when the tile lies in one bin (the common case:
//     bins hold ~10^5 entries), per element otherwise, on order-preserving
//     integer images of the times.
// The bin is computed with bin_of() from t_start exactly as k_keys did (same
// inputs, same arithmetic).
struct GatherSmem {
    unsigned long long s_o0[BT / 32], s_o1[BT / 32];
    uint32_t s_cnt, s_blk;
};

// The tile's records are in registers (r0, r1 for rows id) and its keys in
// s_key[1..] with the halo in s_key[0]: write the SoA streams, then the
// per-cell / per-bin bookkeeping.  Ends with a barrier.
template <int ITEMS>
__device__ __forceinline__ void gather_tile(size_t n, size_t p0, const uint32_t (&id)[ITEMS],
                                            const double4 (&r0)[ITEMS],
                                            const double4 (&r1)[ITEMS], SegSoA& soa,
                                            const GridParams& g, uint32_t* __restrict__ bin_start,
                                            unsigned long long* __restrict__ bin_t0min,
                                            unsigned long long* __restrict__ bin_t1max,
                                            unsigned long long* __restrict__ count,
                                            const unsigned long long* s_key, int32_t* s_bin,
                                            GatherSmem& sm, bool key_bins,
                                            const uint32_t* __restrict__ orows,
                                            uint32_t* __restrict__ obits) {
    unsigned long long o0 = ~0ull, o1 = 0ull;
    unsigned long long e0[ITEMS], e1[ITEMS];   // time extent each position gives its bin
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const size_t p = p0 + (size_t)k * BT + threadIdx.x;
        if (p < n) {
            const double4 s0 = r0[k], s1 = r1[k];
            const double dur = s1.x - s0.x;
            // three correctly rounded divisions, not one reciprocal and
            // three products: equal ratios must give equal velocities, or a
            // pair of coincident segments at d = 0 (no relative motion, the
            // whole overlap within d) degenerates to a single instant
            soa.store4(p, make_double2(s0.x, s1.x), make_double2(s0.y, velocity(s0.y, s1.y, dur)),
                       make_double2(s0.z, velocity(s0.z, s1.z, dur)),
                       make_double2(s0.w, velocity(s0.w, s1.w, dur)));
            soa.eid[p] = id[k];
            // (with outlier copies a position's bin is its key's: a copy is
            // filed in every bin its time spans, not only its start's)
            const int32_t bk = key_bins ? (int32_t)(s_key[1 + k * BT + threadIdx.x] / g.cells_per_bin)
                                        : bin_of(g, s0.x);
            s_bin[1 + k * BT + threadIdx.x] = bk;
            double ta = s0.x, tb = s1.x;
            const bool copy = orows && ((__ldg(orows + (id[k] >> 5)) >> (id[k] & 31u)) & 1u);
            if (copy) {
                // an outlier's copy stands for its time inside this bin only
                if (bk != bin_of(g, s0.x)) ta = fmax(ta, g.tmin + (double)bk * g.b);
                if (bk != bin_of(g, s1.x)) tb = fmin(tb, g.tmin + (double)(bk + 1) * g.b);
            }
            // bitmap of the positions holding copies (32 consecutive
            // positions per warp and k: one ballot, one word)
            if (obits) {
                const uint32_t w = __ballot_sync(__activemask(), copy);
                if ((threadIdx.x & 31) == 0) obits[p >> 5] = w;
            }
            const unsigned long long a = ordered_bits(ta), b = ordered_bits(tb);
            e0[k] = a;
            e1[k] = b;
            o0 = a < o0 ? a : o0;
            o1 = b > o1 ? b : o1;
        } else {
            e0[k] = ~0ull;
            e1[k] = 0ull;
        }
    }
    __syncthreads();
    const int32_t bfirst = s_bin[1];
    bool one_bin = true;
    uint32_t cells = 0, blks = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const int loc = k * BT + threadIdx.x;
        const size_t p = p0 + (size_t)loc;
        if (p < n) {
            cells += (p == 0 || s_key[loc] != s_key[loc + 1]) ? 1u : 0u;
            blks += (p == 0 || (s_key[loc] >> 3) != (s_key[loc + 1] >> 3)) ? 1u : 0u;
            const int32_t bp = s_bin[loc], b = s_bin[loc + 1];
            for (int32_t bb = bp + 1; bb <= b; ++bb) bin_start[bb] = (uint32_t)p;
            if (p == n - 1)
                for (int32_t bb = b + 1; bb <= g.m; ++bb) bin_start[bb] = (uint32_t)n;
            one_bin = one_bin && b == bfirst;
        }
    }
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    cells = __reduce_add_sync(0xffffffffu, cells);
    blks = __reduce_add_sync(0xffffffffu, blks);
    if (lane == 0 && cells) atomicAdd(&sm.s_cnt, cells);
    if (lane == 0 && blks) atomicAdd(&sm.s_blk, blks);
    if (__syncthreads_and(one_bin)) {
#pragma unroll
        for (int off = 16; off; off >>= 1) {
            const unsigned long long x = __shfl_xor_sync(0xffffffffu, o0, off);
            const unsigned long long y = __shfl_xor_sync(0xffffffffu, o1, off);
            o0 = x < o0 ? x : o0;
            o1 = y > o1 ? y : o1;
        }
        if (lane == 0) { sm.s_o0[warp] = o0; sm.s_o1[warp] = o1; }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int w = 1; w < BT / 32; ++w) {
                o0 = sm.s_o0[w] < o0 ? sm.s_o0[w] : o0;
                o1 = sm.s_o1[w] > o1 ? sm.s_o1[w] : o1;
            }
            atomicMin(&bin_t0min[bfirst], o0);
            atomicMax(&bin_t1max[bfirst], o1);
        }
    } else {                                           // tile spans bins: per element
#pragma unroll
        for (int k = 0; k < ITEMS; ++k) {
            const int loc = k * BT + threadIdx.x;
            if (p0 + (size_t)loc < n) {
                const int32_t b = s_bin[loc + 1];
                atomicMin(&bin_t0min[b], e0[k]);
                atomicMax(&bin_t1max[b], e1[k]);
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && sm.s_cnt) {         // count[0]: cells, count[1]: blocks of 8 keys
        atomicAdd(count, (unsigned long long)sm.s_cnt);
        atomicAdd(count + 1, (unsigned long long)sm.s_blk);
    }
}

template <int ITEMS, int MINB = 4>
__global__ void __launch_bounds__(BT, MINB) k_gather_cells(const double4* __restrict__ D, size_t n,
                                                    const SortedKeys sk, SegSoA soa, GridParams g,
                                                    uint32_t* __restrict__ bin_start,
                                                    unsigned long long* __restrict__ bin_t0min,
                                                    unsigned long long* __restrict__ bin_t1max,
                                                    unsigned long long* __restrict__ count,
                                                    int key_bins,
                                                    const uint32_t* __restrict__ orows,
                                                    uint32_t* __restrict__ obits) {
    constexpr int TILE = BT * ITEMS;
    __shared__ unsigned long long s_key[TILE + 1];
    __shared__ int32_t s_bin[TILE + 1];
    __shared__ GatherSmem sm;
    const size_t p0 = (size_t)blockIdx.x * TILE;
    uint32_t id[ITEMS];
    double4 r0[ITEMS], r1[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const size_t p = p0 + (size_t)k * BT + threadIdx.x;
        if (p < n) {
            id[k] = sk.row(p);
            s_key[1 + k * BT + threadIdx.x] = sk.key(p);
        } else {
            id[k] = 0u;
        }
    }
    if (threadIdx.x == 0) {
        sm.s_cnt = 0;
        sm.s_blk = 0;
        if (p0 > 0) {                                  // halo: sorted position p0 - 1
            // keys are bin-major (key = bin * cells_per_bin + cell), so the
            // halo's bin needs no dependent load of its record
            const unsigned long long hk = sk.key(p0 - 1);
            s_key[0] = hk;
            s_bin[0] = (int32_t)(hk / g.cells_per_bin);
        } else {
            s_key[0] = ~0ull;
            s_bin[0] = -1;
        }
    }
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        const size_t p = p0 + (size_t)k * BT + threadIdx.x;
        if (p < n) {
            r0[k] = ld256(D + 2 * (size_t)id[k]);
            r1[k] = ld256(D + 2 * (size_t)id[k] + 1);
        }
    }
    gather_tile<ITEMS>(n, p0, id, r0, r1, soa, g, bin_start, bin_t0min, bin_t1max, count, s_key,
                       s_bin, sm, key_bins != 0, orows, obits);
}


__global__ void k_fill_u64(unsigned long long* __restrict__ a, size_t n, unsigned long long v) {
    size_t i = (size_t)blockIdx.x * BT + threadIdx.x;
    if (i < n) a[i] = v;
}

__global__ void k_ordered_to_double(unsigned long long* __restrict__ a, size_t n) {
    size_t i = (size_t)blockIdx.x * BT + threadIdx.x;
    if (i < n) {
        double v = from_ordered_bits(a[i]);
        a[i] = (unsigned long long)__double_as_longlong(v);
    }
}


inline unsigned grid_for(size_t n) { return (unsigned)((n + BT - 1) / BT); }

// SMs x resident CTAs of BT threads for kernel f on the current device (one
// full wave for a grid-stride kernel).
int resident_grid(const void* f) {
    int dev = 0, sms = 0, occ = 0;
    DTS_CUDA(cudaGetDevice(&dev));
    DTS_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    DTS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, f, BT, 0));
    return std::max(1, sms * std::max(1, occ));
}

// ---------------------------------------------------------- subbins (ST)
// Coordinate A of a segment's start (row 0) / end (row 1).
template <int A>
__device__ __forceinline__ double coord(const double4& r) {
    return A == 0 ? r.y : (A == 1 ? r.z : r.w);
}

// Number of subbins of dimension a that the entry at sorted position p
// overlaps (its extent [min, max] in a: at most 2 when subbins are
// wider than the largest extent).
template <int A>
__global__ void __launch_bounds__(BT) k_sb_count(const double4* __restrict__ D,
                                                const uint32_t* __restrict__ eid, size_t n,
                                                SubbinIndex sb, uint32_t* __restrict__ cnt) {
    size_t p = (size_t)blockIdx.x * BT + threadIdx.x;
    if (p >= n) return;
    const uint32_t i = eid[p];
    const double c0 = coord<A>(D[2 * (size_t)i]), c1 = coord<A>(D[2 * (size_t)i + 1]);
    cnt[p] = (uint32_t)(subbin_of(sb, A, fmax(c0, c1)) - subbin_of(sb, A, fmin(c0, c1)) + 1);
}

// One (key = subbin * m + bin, value = p) pair per overlapped subbin.
template <int A>
__global__ void __launch_bounds__(BT) k_sb_emit(const double4* __restrict__ D,
                                               const uint32_t* __restrict__ eid,
                                               const SegSoA soa, size_t n,
                                               SubbinIndex sb, GridParams g,
                                               const unsigned long long* __restrict__ off,
                                               unsigned long long* __restrict__ keys,
                                               uint32_t* __restrict__ vals) {
    size_t p = (size_t)blockIdx.x * BT + threadIdx.x;
    if (p >= n) return;
    const uint32_t i = eid[p];
    const double c0 = coord<A>(D[2 * (size_t)i]), c1 = coord<A>(D[2 * (size_t)i + 1]);
    const int32_t jlo = subbin_of(sb, A, fmin(c0, c1)), jhi = subbin_of(sb, A, fmax(c0, c1));
    const unsigned long long bin = (unsigned long long)bin_of(g, __ldg(soa.at(p)).x);
    unsigned long long o = off[p];
    for (int32_t j = jlo; j <= jhi; ++j, ++o) {
        keys[o] = (unsigned long long)j * (unsigned long long)g.m + bin;
        vals[o] = (uint32_t)p;
    }
}

__global__ void __launch_bounds__(BT) k_map_ids(uint32_t* __restrict__ eid, size_t n,
                                               const uint32_t* __restrict__ emap) {
    size_t p = (size_t)blockIdx.x * BT + threadIdx.x;
    if (p < n) eid[p] = emap[eid[p]];
}

__global__ void __launch_bounds__(BT) k_gather_u32(uint32_t* __restrict__ out,
                                                  const uint32_t* __restrict__ in,
                                                  const uint32_t* __restrict__ rows, size_t n) {
    size_t p = (size_t)blockIdx.x * BT + threadIdx.x;
    if (p < n) out[p] = in[rows[p]];
}

// dir[k] = first position of key >= k in the sorted keys, k in [0, nkeys].
__global__ void __launch_bounds__(BT) k_sb_dir(const unsigned long long* __restrict__ keys,
                                              size_t len, unsigned long long nkeys,
                                              uint32_t* __restrict__ dir) {
    size_t q = (size_t)blockIdx.x * BT + threadIdx.x;
    if (q >= len) return;
    const long long k = (long long)keys[q];
    const long long kp = q == 0 ? -1 : (long long)keys[q - 1];
    for (long long kk = kp + 1; kk <= k; ++kk) dir[kk] = (uint32_t)q;
    if (q == len - 1)
        for (long long kk = k + 1; kk <= (long long)nkeys; ++kk) dir[kk] = (uint32_t)len;
}

}  // namespace

// GPUSpatioTemporal index (P:L86-P:L92), built on the device over the sorted
// entries: per dimension, (subbin, bin) keys for every overlap, a stable
// radix sort (positions stay ascending inside a chunk) and a directory of
// chunk offsets.
// rec[j] = the record at sorted position ids[j] (two 256-bit accesses).
__global__ void __launch_bounds__(BT) k_sb_gather_rec(double4* __restrict__ rec, const SegSoA soa,
                                                     const uint32_t* __restrict__ ids,
                                                     unsigned long long len) {
    const unsigned long long j = (unsigned long long)blockIdx.x * BT + threadIdx.x;
    if (j >= len) return;
    double2 st, sx, sy, sz;
    soa.load4(__ldg(ids + j), st, sx, sy, sz);
    double* r = reinterpret_cast<double*>(rec + 2 * j);
    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(r), "d"(st.x), "d"(st.y),
                 "d"(sx.x), "d"(sx.y) : "memory");
    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(r + 4), "d"(sy.x), "d"(sy.y),
                 "d"(sz.x), "d"(sz.y) : "memory");
}

static void build_subbins(dts_index* idx, const double4* D, size_t n, const Bounds& hb,
                          const dts_index_params& p, cudaStream_t s) {
    const GridParams& g = idx->gp;
    SubbinIndex& sb = idx->sb;
    const int32_t vreq = p.subbins > 0 ? (int32_t)std::min<uint32_t>(p.subbins, 1u << 16) : 16;
    sb.m = g.m;
    for (int a = 0; a < 3; ++a) {
        const double span = hb.hi[a] - hb.lo[a];
        int32_t v = vreq;
        if (hb.ext[a] > 0.0) v = (int32_t)std::min<double>(v, std::max(1.0, std::floor(span / hb.ext[a])));
        if (!(span > 0.0)) v = 1;
        sb.v[a] = v;
        sb.o[a] = hb.lo[a];
        sb.inv_w[a] = span > 0.0 ? (double)v / span : 0.0;
    }
    for (int a = 0; a < 3; ++a) {
        DevBuf<uint32_t> cnt(n, s);
        DevBuf<unsigned long long> off(n + 1, s);
        if (a == 0) k_sb_count<0><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, n, sb, cnt.p);
        else if (a == 1) k_sb_count<1><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, n, sb, cnt.p);
        else k_sb_count<2><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, n, sb, cnt.p);
        DTS_LAUNCH_CHECK();
        scan_exclusive_u32_to_u64(cnt.p, off.p, n, s);
        unsigned long long len = 0;
        DTS_CUDA(cudaMemcpyAsync(&len, off.p + n, sizeof(len), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        if (len >= (1ull << 32)) throw Error(DTS_ENOTSUP, "subbin id array exceeds 2^32 entries");
        const unsigned long long nkeys = (unsigned long long)sb.v[a] * (unsigned long long)g.m;
        DevBuf<unsigned long long> keys(len, s), keys_tmp(len, s);
        DevBuf<uint32_t> vals_tmp(len, s);
        uint32_t* blk = static_cast<uint32_t*>(cache_alloc((len + nkeys + 1) * sizeof(uint32_t)));
        idx->sb_block[a] = blk;
        idx->sb_len[a] = len;
        if (a == 0)
            k_sb_emit<0><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, idx->soa, n, sb, g,
                                                    off.p, keys.p, blk);
        else if (a == 1)
            k_sb_emit<1><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, idx->soa, n, sb, g,
                                                    off.p, keys.p, blk);
        else
            k_sb_emit<2><<<grid_for(n), BT, 0, s>>>(D, idx->soa.eid, idx->soa, n, sb, g,
                                                    off.p, keys.p, blk);
        DTS_LAUNCH_CHECK();
        radix_sort_pairs(keys.p, blk, keys_tmp.p, vals_tmp.p, len, bits_for(nkeys - 1), s);
        k_sb_dir<<<grid_for(len), BT, 0, s>>>(keys.p, len, nkeys, blk + len);
        DTS_LAUNCH_CHECK();
        sb.ids[a] = blk;
        sb.dir[a] = blk + len;
        // the records of the id array, in its order (B200 layout choice: the
        // paper's X/Y/Z arrays hold ids; a copy of the 64-byte records
        // per dimension turns each candidate into a contiguous read)
        double4* rec = static_cast<double4*>(cache_alloc((size_t)len * 2 * sizeof(double4) + 64));
        idx->sb_rec[a] = rec;
        if (len) {
            k_sb_gather_rec<<<grid_for(len), BT, 0, s>>>(rec, idx->soa, blk, len);
            DTS_LAUNCH_CHECK();
        }
        sb.rec[a] = rec;
        DTS_CUDA(cudaStreamSynchronize(s));
    }
}

// Host-side choice of the temporal bins and spatial cells.
// Cell width per axis = (max extent + d_hint) x scale, with scale 0.5 for x
// and 1 for y and z: x is the contiguous axis of the key, so a stencil row
// costs one probe (one or two 8-cell blocks) whatever its x-cell count, and
// narrower x cells only drop candidates.  Measured (search only, index
// resident, B200): C4 pass 1 0.612 -> 0.574 ms (32.1 M -> 25.9 M candidates),
// C2 d = 8 4.30 -> 3.71, C3 d = 5 0.088 -> 0.070; the small sets (C1, S1,
// C2 d = 0.09) within +-0.01 ms.  Finer y or z cells add rows (probes) and
// measured slower.  DTS_CELL_SCALE="sx,sy,sz" overrides (any width gives
// the same results: the stencil covers as many cells as it needs).
static double cell_scale(int a) {
    static const std::vector<double> f = [] {
        std::vector<double> v{0.5, 1.0, 1.0};
        const char* e = getenv("DTS_CELL_SCALE");
        if (e) sscanf(e, "%lf,%lf,%lf", &v[0], &v[1], &v[2]);
        for (double& x : v) if (!(x > 0.0) || !std::isfinite(x)) x = 1.0;
        return v;
    }();
    return f[a];
}

static void choose_grid(const Bounds& b, const dts_index_params& p, GridParams& g, size_t n,
                        double occ, bool* capped = nullptr) {
    if (capped) *capped = false;
    const double span_t = b.tmax - b.tmin;
    g.tmin = b.tmin;
    g.maxdur = b.maxdur;
    const uint64_t MAXBINS = 1u << 22;
    double bw;
    if (p.temporal_bins > 0 && span_t > 0.0) bw = span_t / (double)p.temporal_bins;
    else bw = b.maxdur;                               // one bin per max duration
    if (!(bw > 0.0) || !std::isfinite(bw)) bw = span_t > 0.0 ? span_t : 1.0;
    double mb = std::floor(span_t / bw) + 1.0;
    if (mb > (double)MAXBINS) { bw = span_t / (double)(MAXBINS - 1); mb = (double)MAXBINS; }
    g.b = bw;
    g.inv_b = 1.0 / bw;
    g.m = (int32_t)mb;

    const double MAXC = (double)(1u << 20);
    for (int a = 0; a < 3; ++a) {
        const double span = b.hi[a] - b.lo[a];
        double w = b.ext[a] + (p.d_hint > 0.0 ? p.d_hint : 0.0);
        if (p.cells_per_dim > 0) w = std::max(w, span / (double)p.cells_per_dim);
        // temporal and subbin methods use one cell per bin: the sort key is the
        // bin, so entries are grouped by t_start bin as in P:L76
        if (p.method != DTS_METHOD_GRID) w = std::max(span, 1.0) * 2.0;
        else w *= cell_scale(a);
        w = std::max(w, span / (MAXC - 1.0));
        w = std::max(w, 1e-12 * b.absmax);
        if (!(w > 0.0) || !std::isfinite(w)) w = 1.0;
        g.o[a] = b.lo[a];
        g.w[a] = w;
        g.half_ext[a] = 0.5 * b.ext[a];
        g.nc[a] = (int32_t)std::min(std::floor(span / w) + 1.0, MAXC);
    }
    // sparse data: cap the cells per bin at 1024 x the entries per bin per
    // occupied fraction of the box (C3, 384 entries per bin in a 1000^3
    // cube, had 12.7 M cells per bin: 96 row probes per query, nearly all
    // empty); clustered or dense data (C4: 26 cells per such entry) are left
    // alone.  Widths only grow, so the E + d lower bound still holds.
    static const double dcap = [] {          // DTS_DENSITY_CAP: 0 disables
        const char* e = getenv("DTS_DENSITY_CAP");
        return e ? atof(e) : 1024.0;
    }();
    if (p.method == DTS_METHOD_GRID && p.cells_per_dim == 0 && occ > 0.0 && dcap > 0.0 && n > 0) {
        const double nb = (double)n / (double)g.m;
        const double cap = std::max(64.0, dcap * nb / occ);
        const double prod = (double)g.nc[0] * g.nc[1] * g.nc[2];
        if (prod > cap) {
            if (capped) *capped = true;
            const double f = std::cbrt(prod / cap);
            for (int a = 0; a < 3; ++a) {
                const double span = b.hi[a] - b.lo[a];
                g.w[a] *= f;
                g.nc[a] = (int32_t)std::min(std::floor(span / g.w[a]) + 1.0, MAXC);
            }
        }
    }
    // a row's x-cells start at a multiple of 8 keys: nc[0] is rounded up to a
    // multiple of 8 (the extra cells stay empty), so an 8-key hash block never
    // straddles two rows or two bins.  A block holding more than 65535 entries
    // is returned whole by a row probe (superset); if it could straddle rows,
    // two probes of one query would return the same entries twice.
    // (the temporal and subbin methods never probe cells: one cell per bin)
    const bool grid = p.method == DTS_METHOD_GRID;
    auto round8 = [grid](int32_t v) { return grid ? (int32_t)(((int64_t)v + 7) / 8 * 8) : v; };
    g.nc[0] = round8(g.nc[0]);
    // keep the key space below 2^62: coarsen the finest axis until it fits
    while ((double)g.m * g.nc[0] * g.nc[1] * g.nc[2] >= 4.6e18) {
        int a = 0;
        for (int j = 1; j < 3; ++j) if (g.nc[j] > g.nc[a]) a = j;
        g.w[a] *= 2.0;
        g.nc[a] = (int32_t)std::floor((b.hi[a] - b.lo[a]) / g.w[a]) + 1;
        if (a == 0) g.nc[0] = round8(g.nc[0]);
    }
    for (int a = 0; a < 3; ++a) g.inv_w[a] = 1.0 / g.w[a];
    g.cells_per_bin = (unsigned long long)g.nc[0] * g.nc[1] * g.nc[2];
}

void build_index_device(dts_index* idx, const dts_segment* D_dev, size_t n,
                        const dts_index_params& p, cudaStream_t s) {
    idx->n = n;
    idx->eid_bits = p.entry_ids ? 32 : std::max(1, bits_for(n ? n - 1 : 0));
    if (n == 0) return;
    const double4* D = reinterpret_cast<const double4*>(D_dev);
    // phase events: start, bounds, keys, sort, gather, insert (+ end)
    // (kept in the index: the build returns without waiting for its last
    //  kernels, the times are read by dts_index_get_info)
    struct Events {
        cudaEvent_t ev[7];
        bool keep = false;
        Events() { for (auto& e : ev) DTS_CUDA(cudaEventCreate(&e)); }
        ~Events() { if (!keep) for (auto& e : ev) cudaEventDestroy(e); }
    } evs;
    cudaEvent_t* ev = evs.ev;
    int nev = 0;
    // (at most 7 marks; a retried phase keeps its first mark)
    auto mark = [&] { if (nev < 7) DTS_CUDA(cudaEventRecord(ev[nev++], s)); };
    mark();

    const int np = (int)std::min<size_t>(grid_for(n), 148 * 8);
    DevBuf<Bounds> partial(np, s), total(1, s);
    const int row_bits = std::max(1, bits_for(n - 1));
    static const bool allow_packed = [] {       // DTS_PACKED_SORT=0: (key, id) pairs
        const char* e = getenv("DTS_PACKED_SORT");
        return !(e && e[0] == '0');
    }();
    static const bool allow_fused = [] {        // DTS_FUSED_KEYS=0: bounds, then keys
        const char* e = getenv("DTS_FUSED_KEYS");
        return !(e && e[0] == '0');
    }();
    auto check = [](const Bounds& b) {
        if (b.bad & 1) throw Error(DTS_EINVAL, "entry segment with a non-finite coordinate or time");
        if (b.bad & 2) throw Error(DTS_EINVAL, "entry segment with t_end < t_start");
        if (b.bad & 4) throw Error(DTS_EINVAL, "entry segment whose speed overflows fp64");
    };
    auto key_bits_of = [](const GridParams& g) {
        return bits_for((unsigned long long)g.m * g.cells_per_bin - 1ull);
    };
    // pinned landing slot of the exact bounds (read while the sort runs)
    struct BoundsOut {
        Bounds b;
    };
    static thread_local BoundsOut* hb_pinned = [] {
        BoundsOut* q = nullptr;
        DTS_CUDA(cudaMallocHost(&q, sizeof(BoundsOut)));
        return q;
    }();

    Bounds hb;
    GridParams g{};
    DevBuf<unsigned long long> keys(n, s), keys_tmp(n, s);
    // long-segment outliers (internal.cuh "outliers"): rows flagged by the
    // fused pass, filed as copies along their path; nt = sorted positions
    static const bool outliers_on = [] {     // DTS_OUTLIERS=0: plain filing
        const char* e = getenv("DTS_OUTLIERS");
        return !(e && e[0] == '0');
    }();
    Thresh th{{0, 0, 0}, 0, 0};
    DevBuf<uint32_t> orows(0, s), olist(0, s);
    DevBuf<unsigned int> ocount(0, s);
    size_t nt = n;
    unsigned long long n_out = 0;
    DevBuf<uint32_t> ids(0, s), ids_tmp(0, s);
    SortedKeys sk;
    bool done = false;
    // sample occupancy of the bounding box (choose_grid's density cap)
    double occ = -1.0;
    DevBuf<uint32_t> occ_bits(OCC_RES * OCC_RES * OCC_RES / 32, s);
    static thread_local uint32_t* occ_host = [] {
        uint32_t* q = nullptr;
        DTS_CUDA(cudaMallocHost(&q, OCC_RES * OCC_RES * OCC_RES / 8));
        return q;
    }();
    auto occ_launch = [&](size_t S, const Bounds* bnd) {
        DTS_CUDA(cudaMemsetAsync(occ_bits.p, 0, OCC_RES * OCC_RES * OCC_RES / 8, s));
        const int nb = (int)std::min<size_t>(std::max<size_t>(grid_for(S) / 4, 1), 592);
        k_sample_occupancy<<<nb, BT, 0, s>>>(D, n, S, bnd, occ_bits.p);
        DTS_LAUNCH_CHECK();
        DTS_CUDA(cudaMemcpyAsync(occ_host, occ_bits.p, OCC_RES * OCC_RES * OCC_RES / 8,
                                 cudaMemcpyDeviceToHost, s));
    };
    auto occ_fraction = [&]() {
        size_t c = 0;
        for (int i = 0; i < OCC_RES * OCC_RES * OCC_RES / 32; ++i) c += __builtin_popcount(occ_host[i]);
        return (double)c / (double)(OCC_RES * OCC_RES * OCC_RES);
    };
    if (allow_fused && allow_packed && radix_onesweep(n)) {
        // 1. bounds of a strided sample -> provisional grid.  Any grid gives
        //    the same results: the keys only group the entries, and every
        //    query stencil is derived from the EXACT max extent and duration
        //    (half_ext, maxdur set below), with cell_of/bin_of clamping
        //    entries outside the sampled domain into the boundary cells and
        //    bins, a monotone map, so the stencil stays a superset.
        static const int slog = [] {            // DTS_SAMPLE_LOG2: sample size
            const char* e = getenv("DTS_SAMPLE_LOG2");
            return e ? std::max(10, std::min(24, atoi(e))) : 16;
        }();
        const size_t S = std::min<size_t>(n, (size_t)1 << slog);
        const int nps = (int)std::min<size_t>(std::max<size_t>(grid_for(S) / 4, 1), 592);
        const bool want_out = outliers_on && p.method == DTS_METHOD_GRID;
        // the outlier list's buffers do not depend on the sample: allocated
        // before the host waits for it
        if (want_out) {
            orows.alloc(n / 32 + 1, s);
            olist.alloc(std::min<size_t>(n, (size_t)(n / 64) + 4096), s);
            ocount.alloc(1, s);
            DTS_CUDA(cudaMemsetAsync(orows.p, 0, (n / 32 + 1) * 4, s));
            DTS_CUDA(cudaMemsetAsync(ocount.p, 0, 4, s));
        }
        DevBuf<SampleOut> so(1, s);
        k_bounds_sample<<<nps, BT, 0, s>>>(D, n, S, partial.p, nullptr);
        DTS_LAUNCH_CHECK();
        k_bounds_final<<<1, BT, 0, s>>>(partial.p, nps, want_out ? total.p : &so.p->b);
        DTS_LAUNCH_CHECK();
        if (want_out) {
            // thresholds on the device, then the sample's bounds without the
            // outliers; one host round trip for both
            k_thresh<<<1, 1, 0, s>>>(total.p, &so.p->th);
            DTS_LAUNCH_CHECK();
            k_bounds_sample<<<nps, BT, 0, s>>>(D, n, S, partial.p, &so.p->th);
            DTS_LAUNCH_CHECK();
            k_bounds_final<<<1, BT, 0, s>>>(partial.p, nps, &so.p->b);
            DTS_LAUNCH_CHECK();
        } else {
            DTS_CUDA(cudaMemsetAsync(&so.p->th, 0, sizeof(Thresh), s));
        }
        SampleOut hso;
        DTS_CUDA(cudaMemcpyAsync(&hso, so.p, sizeof(SampleOut), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        Bounds hs = hso.b;
        check(hs);
        th = hso.th;
        mark();
        // the occupancy only matters when even a full box would be capped
        // (C3); dense or clustered data (C4, C2, S3) skip its kernel
        bool capped = false;
        choose_grid(hs, p, g, n, 1.0, &capped);
        occ = 1.0;
        if (capped) {
            occ_launch(S, &so.p->b);
            DTS_CUDA(cudaStreamSynchronize(s));
            occ = occ_fraction();
            choose_grid(hs, p, g, n, occ);
        }
        // the fused pass; a second attempt with the exact grid when the
        // sample's grid was far off (the exact path below would drop the
        // outlier filing)
        for (int attempt = 0; attempt < 2 && !done; ++attempt) {
        const int kb = key_bits_of(g);
        if (row_bits + kb <= 64) {
            // 2-3. exact bounds + keys + sort histograms in one read of D
            const PassPlan plan = plan_passes(row_bits, row_bits + kb, true);
            DevBuf<uint32_t> hist((size_t)plan.npass * OS_HSTRIDE, s);
            DTS_CUDA(cudaMemsetAsync(hist.p, 0, (size_t)plan.npass * OS_HSTRIDE * 4, s));
            // grid-stride over D with exactly one wave of resident CTAs
            // (np = 1184 CTAs at 3 per SM left the last of 2.67 waves 2/3 full)
            static const int bk_minb = [] {     // DTS_BK_OCC: CTAs per SM (3: 0.321 ms on C4; 4 spills: 0.355)
                const char* e = getenv("DTS_BK_OCC");
                return (e && e[0] == '4') ? 4 : 3;
            }();
            const int npk = (int)std::min<size_t>((size_t)resident_grid(
                bk_minb == 3 ? (const void*)k_bounds_keys<3, false> : (const void*)k_bounds_keys<4, false>), np);
            OutlierOut oo{};
            if (th.on) {
                if (attempt > 0) {                    // the first attempt's marks
                    DTS_CUDA(cudaMemsetAsync(orows.p, 0, (n / 32 + 1) * 4, s));
                    DTS_CUDA(cudaMemsetAsync(ocount.p, 0, 4, s));
                }
                oo = OutlierOut{orows.p, olist.p, ocount.p, (unsigned int)olist.n};
            }
            if (th.on)
                k_bounds_keys<3, true><<<npk, BT, 0, s>>>(D, n, g, keys.p, row_bits, plan,
                                                          partial.p, hist.p, th, oo);
            else if (bk_minb == 3)
                k_bounds_keys<3, false><<<npk, BT, 0, s>>>(D, n, g, keys.p, row_bits, plan,
                                                           partial.p, hist.p, th, oo);
            else
                k_bounds_keys<4, false><<<npk, BT, 0, s>>>(D, n, g, keys.p, row_bits, plan,
                                                           partial.p, hist.p, th, oo);
            DTS_LAUNCH_CHECK();
            k_bounds_final<<<1, BT, 0, s>>>(partial.p, npk, total.p);
            DTS_LAUNCH_CHECK();
            DTS_CUDA(cudaMemcpyAsync(&hb_pinned->b, total.p, sizeof(Bounds), cudaMemcpyDeviceToHost, s));
            cudaEvent_t eb;
            DTS_CUDA(cudaEventCreateWithFlags(&eb, cudaEventDisableTiming));
            DTS_CUDA(cudaEventRecord(eb, s));
            if (attempt == 0) mark();
            // 4. sort, enqueued before the host looks at the outlier count
            //    and the exact bounds (with outliers the keys and their copies
            //    are sorted again below, from a snapshot of the digit counts)
            DevBuf<uint32_t> hist0(th.on ? (size_t)plan.npass * OS_HSTRIDE : 0, s);
            if (th.on)
                DTS_CUDA(cudaMemcpyAsync(hist0.p, hist.p, (size_t)plan.npass * OS_HSTRIDE * 4,
                                         cudaMemcpyDeviceToDevice, s));
            unsigned long long* sorted = radix_sort_keys_hist(keys.p, keys_tmp.p, n, plan, hist.p, s);
            bool drop_outliers = false;
            if (th.on) {
                // outliers found: their copies join the keys before the sort
                // (the host needs their number first)
                DTS_CUDA(cudaEventSynchronize(eb));
                const unsigned long long nout = hb_pinned->b.nout;
                if (nout > (unsigned long long)olist.n) {
                    drop_outliers = true;          // too many to be outliers: plain filing
                } else if (nout > 0) {
                    DevBuf<uint32_t> cnt(nout, s);
                    DevBuf<unsigned long long> off(nout + 1, s);
                    k_outlier_count<<<grid_for(nout), BT, 0, s>>>(D, olist.p, (uint32_t)nout, g,
                                                                  cnt.p);
                    DTS_LAUNCH_CHECK();
                    scan_exclusive_u32_to_u64(cnt.p, off.p, nout, s);
                    unsigned long long ncp = 0;
                    DTS_CUDA(cudaMemcpyAsync(&ncp, off.p + nout, 8, cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                    if (ncp > std::min<unsigned long long>(8ull * n + (1ull << 20), 1ull << 27) ||
                        n + ncp >= (1ull << 32)) {
                        drop_outliers = true;
                    } else {
                        DevBuf<unsigned long long> k2(n + ncp, s), k2t(n + ncp, s);
                        // (the keys in any order: the sort's result is unique)
                        DTS_CUDA(cudaMemcpyAsync(k2.p, sorted, n * 8, cudaMemcpyDeviceToDevice, s));
                        k_outlier_emit<<<grid_for(nout), BT, 0, s>>>(D, olist.p, (uint32_t)nout, g,
                                                                     off.p, k2.p + n, row_bits,
                                                                     plan, hist0.p);
                        DTS_LAUNCH_CHECK();
                        keys.release();
                        keys_tmp.release();
                        keys.p = k2.detach(); keys.n = n + ncp; keys.s = s;
                        keys_tmp.p = k2t.detach(); keys_tmp.n = n + ncp; keys_tmp.s = s;
                        nt = n + ncp;
                        n_out = nout;
                        sorted = radix_sort_keys_hist(keys.p, keys_tmp.p, nt, plan, hist0.p, s);
                    }
                }
            }
            if (!drop_outliers) {
                sk.a = sorted;
                sk.shift = row_bits;
                sk.ids = nullptr;
            }
            DTS_CUDA(cudaEventSynchronize(eb));
            cudaEventDestroy(eb);
            hb = hb_pinned->b;
            check(hb);
            // keep the provisional grid unless the sample missed the extents
            // badly (cells or bins far narrower or wider than the exact rule
            // gives: correct either way, only slower)
            GridParams gf{};
            choose_grid(hb, p, gf, n, occ);
            bool ok = g.b >= 0.75 * gf.b && g.b <= 1.5 * gf.b;
            for (int a = 0; a < 3; ++a) ok = ok && g.w[a] >= 0.75 * gf.w[a] && g.w[a] <= 1.5 * gf.w[a];
            // ... or missed more than a tenth of the time range: entries
            // starting outside it are clamped into the end bins (a sample of
            // one time step made two bins of 193 on a trajectory-major
            // input).  Space is not checked: a galaxy's sparse outskirts
            // beyond the sample clamp a few entries, harmlessly.
            {
                const double slack = g.b * std::max(1.0, 0.1 * (double)g.m);
                ok = ok && hb.tmin >= g.tmin - slack && hb.tmax <= g.tmin + (double)g.m * g.b + slack;
            }
            static const bool dbg = getenv("DTS_DEBUG_BUILD") != nullptr;
            if (dbg)
                fprintf(stderr, "[dts build] n=%zu th.on=%d th=(%g %g %g | %g) nout=%llu nt=%zu "
                                "drop=%d ok=%d g.b=%g gf.b=%g g.w=(%g %g %g) gf.w=(%g %g %g)\n",
                        n, th.on, th.ext[0], th.ext[1], th.ext[2], th.dur,
                        (unsigned long long)hb.nout, nt, (int)drop_outliers, (int)ok, g.b, gf.b,
                        g.w[0], g.w[1], g.w[2], gf.w[0], gf.w[1], gf.w[2]);
            if (ok && !drop_outliers) {
                for (int a = 0; a < 3; ++a) g.half_ext[a] = 0.5 * hb.ext[a];
                g.maxdur = hb.maxdur;
                idx->key_bits = kb;
                idx->fused_keys = true;
                done = true;
            } else {
                nt = n;                         // start over (or the exact path below)
                n_out = 0;
                if (drop_outliers || !th.on) break;
                g = gf;                         // retry once with the exact (main) grid
            }
        } else {
            break;
        }
        }
    }
    if (!done) {
        // 1. exact bounds + validation, 2. grid, 3. keys, 4. sort
        k_bounds<<<np, BT, 0, s>>>(D, n, partial.p);
        DTS_LAUNCH_CHECK();
        k_bounds_final<<<1, BT, 0, s>>>(partial.p, np, total.p);
        DTS_LAUNCH_CHECK();
        if (nev == 1) mark();
        DTS_CUDA(cudaMemcpyAsync(&hb, total.p, sizeof(Bounds), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        check(hb);
        g = GridParams{};
        if (occ < 0.0) {            // no sample taken yet: the strided sample's occupancy
            bool capped = false;
            choose_grid(hb, p, g, n, 1.0, &capped);
            occ = 1.0;
            if (capped) {
                occ_launch(std::min<size_t>(n, (size_t)1 << 16), total.p);
                DTS_CUDA(cudaStreamSynchronize(s));
                occ = occ_fraction();
            }
            g = GridParams{};
        }
        choose_grid(hb, p, g, n, occ);
        idx->key_bits = key_bits_of(g);
        const bool packed = allow_packed && row_bits + idx->key_bits <= 64;
        if (!packed) {
            ids.alloc(n, s);
            ids_tmp.alloc(n, s);
        }
        k_keys<<<grid_for(n), BT, 0, s>>>(D, n, g, keys.p, ids.p, row_bits);
        DTS_LAUNCH_CHECK();
        if (nev == 2) mark();
        if (packed) {   // keys-only sort of the key bits; rows ride in the low bits
            sk.a = radix_sort_keys(keys.p, keys_tmp.p, n, row_bits, row_bits + idx->key_bits, s);
            sk.shift = row_bits;
            sk.ids = nullptr;
        } else {
            radix_sort_pairs(keys.p, ids.p, keys_tmp.p, ids_tmp.p, n, idx->key_bits, s);
            ids_tmp.release();
            sk.a = keys.p;
            sk.shift = 0;
            sk.ids = ids.p;
        }
    }
    idx->gp = g;
    for (int a = 0; a < 3; ++a) idx->max_ext[a] = hb.ext[a];

    mark();
    // outliers: the sorted packed keys (cell key << shift | row) and a bitmap
    // of the positions holding copies stay with the index for the search's
    // canonical-copy test
    uint32_t* obits = nullptr;
    if (n_out) {
        const size_t kb8 = nt * sizeof(unsigned long long), rb = (nt / 32 + 1) * sizeof(uint32_t);
        char* ob = static_cast<char*>(cache_alloc(kb8 + rb + 64));
        idx->out_block = ob;
        obits = reinterpret_cast<uint32_t*>(ob + kb8);
        DTS_CUDA(cudaMemsetAsync(obits, 0, rb, s));
        idx->out.okeys = reinterpret_cast<const unsigned long long*>(ob);
        idx->out.obits = obits;
        idx->out.shift = sk.shift;
    }
    // 5. gather into the sorted record layout
    const size_t bytes_soa = nt * (4 * sizeof(double2) + sizeof(uint32_t));
    const size_t bytes_bins = 2 * (size_t)g.m * sizeof(double) + ((size_t)g.m + 1) * 4 + 16;
    char* blk = nullptr;
    blk = static_cast<char*>(cache_alloc(bytes_soa + bytes_bins + 256));
    idx->block = blk;
    idx->soa.rec = reinterpret_cast<double2*>(blk);
    idx->bin_t0min = reinterpret_cast<double*>(idx->soa.rec + 4 * nt);
    idx->bin_t1max = idx->bin_t0min + g.m;
    idx->soa.eid = reinterpret_cast<uint32_t*>(idx->bin_t1max + g.m);
    idx->bin_start = idx->soa.eid + nt;
    unsigned long long* b0 = reinterpret_cast<unsigned long long*>(idx->bin_t0min);
    unsigned long long* b1 = reinterpret_cast<unsigned long long*>(idx->bin_t1max);
    k_fill_u64<<<grid_for(g.m), BT, 0, s>>>(b0, g.m, ~0ull);
    DTS_LAUNCH_CHECK();
    k_fill_u64<<<grid_for(g.m), BT, 0, s>>>(b1, g.m, 0ull);
    DTS_LAUNCH_CHECK();
    // 6. non-empty cells -> hash table of >= 2x as many slots (power of two)
    // (measured: inserting from the gather, with the cells counted first,
    //  costs 1.98 ms against 0.78 + 0.56 ms for gather + separate insert)
    DevBuf<unsigned long long> ncell(2, s);       // cells, blocks of 8 keys
    DTS_CUDA(cudaMemsetAsync(ncell.p, 0, 2 * sizeof(unsigned long long), s));
    // (a persistent variant that loads the next tile's keys while the
    //  current records are in flight measured 0.886 ms against 0.775 for one
    //  tile per CTA: fewer resident CTAs hide less of the row latency)
    static const int gvar = [] {        // DTS_GATHER (C4): 1 (1 entry/thread, 6 CTAs/SM) 0.761 ms,
        const char* e = getenv("DTS_GATHER");   // 2 (2, 4: default) 0.751, 4 (4, 2) 0.751
        return e ? atoi(e) : 2;
    }();
    if (gvar == 1)
        k_gather_cells<1, 6><<<grid_for(nt), BT, 0, s>>>(D, nt, sk, idx->soa, g, idx->bin_start,
                                                        b0, b1, ncell.p, n_out ? 1 : 0, n_out ? orows.p : nullptr, obits);
    else if (gvar == 4)
        k_gather_cells<4, 2><<<grid_for((nt + 3) / 4), BT, 0, s>>>(D, nt, sk, idx->soa, g,
                                                                  idx->bin_start, b0, b1, ncell.p,
                                                                  n_out ? 1 : 0,
                                                                  n_out ? orows.p : nullptr, obits);
    else
        k_gather_cells<2><<<grid_for((nt + 1) / 2), BT, 0, s>>>(D, nt, sk, idx->soa, g,
                                                               idx->bin_start, b0, b1, ncell.p,
                                                               n_out ? 1 : 0,
                                                               n_out ? orows.p : nullptr, obits);
    DTS_LAUNCH_CHECK();
    k_ordered_to_double<<<grid_for(2 * (size_t)g.m), BT, 0, s>>>(b0, 2 * (size_t)g.m);
    DTS_LAUNCH_CHECK();
    mark();
    unsigned long long hc[2] = {0, 0};
    DTS_CUDA(cudaMemcpyAsync(hc, ncell.p, sizeof(hc), cudaMemcpyDeviceToHost, s));
    DTS_CUDA(cudaStreamSynchronize(s));
    idx->n_cells = hc[0];
    // 6. the non-empty blocks of 8 keys -> bucketed hash table, one 32-byte
    //    slot per block (prefix counts per cell), 4.5 slots per block, the
    //    table sized exactly (any bucket count).  Measured on C4 (x cells
    //    halved, 5.9 M blocks; pass 1 / insert): 2.5 slots 0.614 / 0.562 ms,
    //    3.3 0.590 / 0.544, 4.5 0.573 / 0.557, 6 0.569 / 0.605; the
    //    power-of-two table it replaced (5.7 slots here) 0.573 / 0.567
    static const double hload = [] {          // DTS_HASH_SLOTS: slots per block
        const char* e = getenv("DTS_HASH_SLOTS");
        return e ? std::max(1.1, atof(e)) : 4.5;
    }();
    const double items = (double)hc[1];
    // buckets of two slots for `hload` slots per block (even, >= 32)
    const unsigned long long nbk =
        std::max<unsigned long long>(32ull, (unsigned long long)std::ceil(hload * items / 2.0));
    if (nbk >= (1ull << 32)) throw Error(DTS_ENOTSUP, "hash table exceeds 2^32 buckets");
    idx->hash_items = hc[1];
    idx->ht.nbuckets = nbk;
    idx->ht.slots = cache_alloc(sizeof(BlockSlot) * 2 * nbk);
    DTS_CUDA(cudaMemsetAsync(idx->ht.slots, 0xFF, sizeof(BlockSlot) * 2 * nbk, s));
    // lane-parallel walks of the staged keys, warp path past 32 entries
    // (warp-cooperative heads for every block: 0.736 ms on C4; one CAS per
    // cell into cell slots: 0.56 ms; these lane walks: 0.435)
    k_insert_blocks_lane<4, 32><<<grid_for((nt + 3) / 4), BT, 0, s>>>(sk, nt, idx->ht);
    DTS_LAUNCH_CHECK();
    idx->n = nt;
    idx->n_outliers = n_out;
    idx->n_copies = nt - n;
    if (n_out)
        DTS_CUDA(cudaMemcpyAsync(idx->out_block, sk.a, nt * sizeof(unsigned long long),
                                 cudaMemcpyDeviceToDevice, s));
    mark();

    // 7. GPUSpatioTemporal subbin arrays (DTS_METHOD_SUBBIN)
    idx->method = p.method;
    if (p.method == DTS_METHOD_SUBBIN) {
        keys.release();
        keys_tmp.release();
        ids.release();
        build_subbins(idx, D, n, hb, p, s);
    }

    // 8. trajectory ids in sorted order (params.entry_traj, device memory here)
    if (p.entry_traj) {
        idx->etraj = static_cast<uint32_t*>(cache_alloc(nt * sizeof(uint32_t)));
        k_gather_u32<<<grid_for(nt), BT, 0, s>>>(idx->etraj, p.entry_traj, idx->soa.eid, nt);
        DTS_LAUNCH_CHECK();
    }

    // 9. reported entry ids of a shard (params.entry_ids, device memory here)
    if (p.entry_ids) {
        k_map_ids<<<grid_for(nt), BT, 0, s>>>(idx->soa.eid, nt, p.entry_ids);
        DTS_LAUNCH_CHECK();
    }

    mark();
    // no wait here: the last kernels may still run when the build returns;
    // searches on other streams wait for `ready` (search_device), and the
    // phase times are read on demand (index_times)
    for (int i = 0; i < 7; ++i) idx->ev[i] = ev[i];
    idx->nev = nev;
    evs.keep = true;
    idx->ready = ev[nev - 1];
}

void index_times(dts_index* idx) {
    if (idx->nev == 0 || idx->timed) return;
    DTS_CUDA(cudaEventSynchronize(idx->ev[idx->nev - 1]));
    DTS_CUDA(cudaEventElapsedTime(&idx->ms_build, idx->ev[0], idx->ev[idx->nev - 1]));
    for (int i = 0; i < 5; ++i) {
        idx->ms_phase[i] = 0.f;
        if (i + 1 < idx->nev) cudaEventElapsedTime(&idx->ms_phase[i], idx->ev[i], idx->ev[i + 1]);
    }
    idx->timed = true;
}

}  // namespace dts
