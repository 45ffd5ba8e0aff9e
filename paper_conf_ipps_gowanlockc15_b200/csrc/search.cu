// search.cu -- the search hot path: query prep, fused candidate streaming +
// fp64 refinement (count pass with staged hits), exact-offset emission, and
// canonical ordering.
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
//     entries, so a CTA's queries and adjacent CTAs read neighbouring cells
//     (L1/L2 reuse) -- the generalisation of "Q sorted by t_start";
//   * a CTA takes a tile of TQ consecutive sorted queries.  Phase A: all
//     (query, bin, cell) probes of the tile are spread over the CTA's threads
//     (bins filtered by their [min t_start, max t_end] extent, the
//     B_start/B_end test of P:L76; a query whose stencil would need more
//     probes than its bins hold entries falls back to the bins' contiguous
//     range, i.e. GPUTemporal's E_k, as GPUSpatioTemporal falls back in
//     P:L96).  Phase B: a block scan flattens all runs into one candidate
//     sequence that the threads stream with four 128-bit loads per candidate;
//   * refinement in fp64 (readings c1-c4, c8), rejecting on cheap tests before
//     any sqrt or divide;
//   * pass 1 counts per query AND stages the tile's hits, sorted by (query,
//     entry id) in shared memory, in a scratch buffer; an exclusive scan of
//     the counts gives exact offsets; pass 2 copies each tile's staged hits to
//     their final positions.  Output is exact-size, canonical (reading c7) and
//     deterministic.  A tile whose hits overflow its staging space is
//     recomputed in pass 2 (warp per query, ballot-ranked writes at the exact
//     offsets) and then sorted per query -- the count-then-scatter fallback.
#include <algorithm>
#include <cstdlib>
#include <vector>

#include "internal.cuh"

namespace dts {
namespace {

constexpr int PT = 256;                 // threads per CTA in warp-per-query kernels
constexpr int PW = PT / 32;
constexpr unsigned long long NONE = ~0ull;

enum : uint32_t { MODE_DEAD = 0, MODE_GRID = 1, MODE_TEMPORAL = 2 };

struct Counters {                       // device-side statistics / flags
    unsigned long long candidates;
    unsigned long long lookups;
    unsigned long long staged;          // staging slots reserved
    unsigned long long spilled;         // spill slots reserved (may exceed the buffer)
    unsigned long long spill_valid;     // first spill slot not written (~0: all written)
    unsigned int max_count;
    unsigned int n_over;                // tiles re-run (spill buffer full)
    unsigned int n_spill;               // tiles whose hits were spilled
    unsigned int n_big;                 // spilled queries longer than a CTA sort
    unsigned int n_cls[3];              // spilled queries for the CTA sorts, by size class
    unsigned int n_skew;                // ... whose ids cluster (radix sort)
    unsigned int bad;
    unsigned int work;                  // dynamic warp-tile counter
    unsigned long long total;           // results (the scan's total, read back with the rest)
    unsigned int n_desc;                // sub-segments of split long segments
    unsigned int n_dskew;               // ... whose ids cluster (radix sort)
    unsigned int n_bigfb;               // long segments left to the device-wide sort
};

// Query in the velocity form used by the refinement.
struct QState {
    double t0, t1;
    double x0, vx, y0, vy, z0, vz;
};

struct Stencil {
    int32_t lb, hb;          // bin range
    int32_t clo[3], cn[3];   // cell range per axis (start, count)
    uint32_t mode;
    uint32_t nlook;          // probes: rows (grid), 1 (single run), 0 (dead)
    uint32_t rstart, rcnt;   // MODE_TEMPORAL: the one run (positions or id-array slots)
    uint32_t rind;           // 0: direct sorted positions; 1 + a: slots of subbin array a
};

// ------------------------------------------------------------- refinement
// compare() of Alg. 1 l.14 for one (query, entry) pair, readings
// c1-c4: strict temporal overlap [ts, te]; relative position
// A(s) = A0 + s W, s = t - ts in [0, L]; |A(s)|^2 - d^2 = aa s^2 + 2 bb s + cc;
// the closed set where it is <= 0, intersected with [0, L].
__device__ __forceinline__ bool refine(const QState& q, const double2 st, const double2 sx,
                                       const double2 sy, const double2 sz, const double d2,
                                       double& t_out0, double& t_out1) {
    // the temporal and the "outside and not approaching" rejections are
    // taken together, after the whole record is used: a branch on the
    // temporal test alone let ptxas sink the record's second 32-byte load
    // behind it (one more dependent memory round trip per candidate)
    const double ts = fmax(q.t0, st.x);
    const double te = fmin(q.t1, st.y);
    const double dq = ts - q.t0, de = ts - st.x;
    const double ax = fma(de, sx.y, sx.x) - fma(dq, q.vx, q.x0);
    const double ay = fma(de, sy.y, sy.x) - fma(dq, q.vy, q.y0);
    const double az = fma(de, sz.y, sz.x) - fma(dq, q.vz, q.z0);
    const double wx = sx.y - q.vx, wy = sy.y - q.vy, wz = sz.y - q.vz;
    const double cc = fma(ax, ax, fma(ay, ay, fma(az, az, -d2)));
    const double bb = fma(ax, wx, fma(ay, wy, az * wz));
    if (!(ts < te) || (cc > 0.0 && bb >= 0.0)) return false;   // no strict overlap, or
                                                                // outside and not approaching
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

// Candidate stencil of a query ("superset" argument):
// entries filed by t_start bin and MBB-midpoint cell can match only if
//   t_start in (q.t0 - maxdur, q.t1)                           (strict overlap)
//   midpoint_a in [qlo_a - d - ext_a/2, qhi_a + d + ext_a/2]    (per axis)
// both widened by a relative 1e-12 slack that covers fp64 rounding of the
// midpoints and of these bounds (monotone floor() keeps the superset).
__device__ __forceinline__ Stencil make_stencil(const GridParams& g, const QState& q,
                                                const double qlo[3], const double qhi[3],
                                                double d, bool live,
                                                const uint32_t* __restrict__ bin_start,
                                                const double* __restrict__ bin_t0min,
                                                const double* __restrict__ bin_t1max,
                                                uint32_t method, const SubbinIndex& sb) {
    Stencil s;
    s.mode = MODE_DEAD;
    s.nlook = 0;
    s.rstart = s.rcnt = s.rind = 0;
    s.lb = s.hb = 0;
    for (int a = 0; a < 3; ++a) { s.clo[a] = 0; s.cn[a] = 1; }
    if (!live) return s;
    const double mt = 1e-12 * (fabs(q.t0) + g.maxdur);
    s.lb = bin_of(g, q.t0 - g.maxdur - mt);
    s.hb = bin_of(g, q.t1);
    // drop end bins whose extent [min t_start, max t_end] (B_start, B_end of
    // P:L76) does not overlap the query strictly: exact comparisons, so no
    // candidate is lost (on synchronised timesteps this removes the previous
    // step's bin, whose segments only touch the query at q.t0)
    // (the end bins' extents and the bin_start values the usual outcomes need
    //  -- each end kept or moved by one bin -- are loaded together: one memory
    //  round trip instead of three dependent ones)
    const int32_t lb0 = s.lb, hb0 = s.hb;
    double l0 = __ldg(&bin_t0min[lb0]), l1 = __ldg(&bin_t1max[lb0]);
    double h0 = __ldg(&bin_t0min[hb0]), h1 = __ldg(&bin_t1max[hb0]);
    const uint32_t bs_l0 = __ldg(&bin_start[lb0]), bs_l1 = __ldg(&bin_start[lb0 + 1]);
    const uint32_t bs_h0 = __ldg(&bin_start[hb0]), bs_h1 = __ldg(&bin_start[hb0 + 1]);
    while (s.lb <= s.hb && !(l0 < q.t1 && l1 > q.t0)) {
        if (++s.lb <= s.hb) { l0 = __ldg(&bin_t0min[s.lb]); l1 = __ldg(&bin_t1max[s.lb]); }
    }
    if (s.lb > s.hb) {
        s.lb = s.hb = 0;
        return s;
    }
    while (s.hb > s.lb && !(h0 < q.t1 && h1 > q.t0)) {
        if (--s.hb > s.lb) { h0 = __ldg(&bin_t0min[s.hb]); h1 = __ldg(&bin_t1max[s.hb]); }
    }
    // the bins' contiguous entry range: GPUTemporal's E_k
    const uint32_t b0 = s.lb == lb0 ? bs_l0 : (s.lb == lb0 + 1 ? bs_l1 : __ldg(&bin_start[s.lb]));
    const uint32_t b1 = s.hb == hb0 ? bs_h1 : (s.hb == hb0 - 1 ? bs_h0 : __ldg(&bin_start[s.hb + 1]));
    const uint32_t T = b1 - b0;
    if (T == 0) return s;                                  // no entry in these bins
    s.mode = MODE_TEMPORAL;
    s.nlook = 1;
    s.rstart = b0;
    s.rcnt = T;
    s.rind = 0;
    if (method == DTS_METHOD_TEMPORAL) return s;
    if (method == DTS_METHOD_SUBBIN) {
        // GPUSpatioTemporal: among the dimensions where [qlo-d, qhi+d]
        // falls in ONE subbin, take the one whose chunk (subbin j, bins
        // lb..hb) -- contiguous in that dimension's id array -- is smallest;
        // entries overlapping subbin j are listed once, so no duplicates.
        // Otherwise fall back to the temporal range.
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const double ms = 1e-12 * (fabs(qlo[a]) + fabs(qhi[a]) + fabs(sb.o[a]) + d);
            const int32_t jlo = subbin_of(sb, a, qlo[a] - d - ms);
            const int32_t jhi = subbin_of(sb, a, qhi[a] + d + ms);
            if (jlo != jhi) continue;
            const uint32_t* dir = sb.dir[a] + (size_t)jlo * (size_t)sb.m;
            const uint32_t c0 = __ldg(dir + s.lb), c1 = __ldg(dir + s.hb + 1);
            if (c1 - c0 < s.rcnt || (s.rind == 0 && c1 - c0 <= s.rcnt)) {
                s.rstart = c0;
                s.rcnt = c1 - c0;
                s.rind = 1 + a;
            }
        }
        return s;
    }
    double ncomb = (double)(s.hb - s.lb + 1);
    int32_t clo[3], cn[3];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        const double ms = 1e-12 * (fabs(qlo[a]) + fabs(qhi[a]) + fabs(g.o[a]) + d + g.half_ext[a]);
        const double r = d + g.half_ext[a] + ms;
        clo[a] = cell_of(g, a, qlo[a] - r);
        cn[a] = cell_of(g, a, qhi[a] + r) - clo[a] + 1;
        ncomb *= (double)cn[a];
    }
    if (ncomb < (double)T) {                               // else probing costs more than scanning
        s.mode = MODE_GRID;
#pragma unroll
        for (int a = 0; a < 3; ++a) { s.clo[a] = clo[a]; s.cn[a] = cn[a]; }
        s.nlook = (uint32_t)(s.hb - s.lb + 1) * (uint32_t)s.cn[1] * (uint32_t)s.cn[2];  // rows
    }
    return s;
}

// Id array of a single-run query: 1 + a -> subbin array of dimension a.
__device__ __forceinline__ const uint32_t* sb_ids(const SubbinIndex& sb, uint32_t ind) {
    return ind == 1 ? sb.ids[0] : (ind == 2 ? sb.ids[1] : sb.ids[2]);
}

// The record at slot j of the subbin array of dimension ind - 1 (its copy
// in id order, SubbinIndex::rec).
__device__ __forceinline__ void sb_load(const SubbinIndex& sb, uint32_t ind, uint32_t j,
                                        double2& st, double2& sx, double2& sy, double2& sz) {
    const double4* r = (ind == 1 ? sb.rec[0] : (ind == 2 ? sb.rec[1] : sb.rec[2])) + 2 * (size_t)j;
    const double4 a = ld256(r), b = ld256(r + 1);
    st = make_double2(a.x, a.y);
    sx = make_double2(a.z, a.w);
    sy = make_double2(b.x, b.y);
    sz = make_double2(b.z, b.w);
}

// Resolve probe `loc` of a query's stencil into one entry run [start,
// start+cnt).  A grid probe is a stencil ROW (bin, cz, cy) over the cells
// cx in [clo0, clo0 + cn0): keys are row-major with x fastest, so the
// non-empty cells of that x range are consecutive in the sorted order and
// form one contiguous run from the first one's start to the last one's end.
// Their hash slots sit in one or two home buckets (bucket_of), read whole.
__device__ __forceinline__ void resolve(const GridParams& g, const HashTable& ht,
                                        const double* __restrict__ bin_t0min,
                                        const double* __restrict__ bin_t1max,
                                        const uint32_t* __restrict__ bin_start, uint32_t mode,
                                        int32_t lb, int32_t hb, const int32_t clo[3],
                                        const int32_t cn[3], double qt0, double qt1, uint32_t loc,
                                        uint32_t rstart, uint32_t rcnt,
                                        uint32_t& start, uint32_t& cnt, uint32_t& probes) {
    start = 0;
    cnt = 0;
    if (mode == MODE_TEMPORAL) {                 // the query's single precomputed run
        start = rstart;
        cnt = rcnt;
        return;
    }
    const uint32_t nzy = (uint32_t)cn[1] * (uint32_t)cn[2];
    const int32_t bin = lb + (int32_t)(loc / nzy);
    const uint32_t r = loc % nzy;
    const int32_t cz = clo[2] + (int32_t)(r / (uint32_t)cn[1]);
    const int32_t cy = clo[1] + (int32_t)(r % (uint32_t)cn[1]);
    // interior bins only: the end bins were checked by make_stencil
    if (bin != lb && bin != hb && !(__ldg(&bin_t0min[bin]) < qt1 && __ldg(&bin_t1max[bin]) > qt0))
        return;
    const unsigned long long key0 = make_key(g, bin, clo[0], cy, cz);
    const unsigned long long kend = key0 + (unsigned long long)cn[0];   // row keys [key0, kend)
    uint32_t first = 0xffffffffu, last = 0;
    // blocks of 8 keys: the row's keys [key0, kend) lie in blocks
    // key0 >> 3 .. (kend - 1) >> 3 of this row only (nc[0] is a multiple of
    // 8), each one 32-byte slot holding the prefix counts of its 8 cells; a
    // bucket is two slots (64 bytes)
    const BlockSlot* slots = ht.blocks();
    for (unsigned long long blk = key0 >> 3; blk <= (kend - 1) >> 3; ++blk) {
        unsigned long long b = bucket_of(blk, ht);
        ++probes;
        while (true) {
            const ulonglong4 h0 = ld256u(slots + 2 * b), h1 = ld256u(slots + 2 * b + 1);
            const bool m0 = h0.x == blk, m1 = h1.x == blk;
            if (m0 || m1) {
                const ulonglong4 h = m0 ? h0 : h1;
                const uint32_t bstart = (uint32_t)h.y, big = (uint32_t)(h.y >> 32);
                const unsigned long long base = blk << 3;
                const uint32_t lo = (uint32_t)((key0 > base ? key0 : base) - base);
                const uint32_t hi = (uint32_t)(((kend - 1) < base + 7 ? (kend - 1) : base + 7) - base);
                uint32_t s0, s1;
                if (big) {                       // the whole block (superset)
                    s0 = bstart;
                    s1 = bstart + (uint32_t)h.z;
                } else {                         // cum[j]: 16 bits at word z (j < 4) or w
                    const uint32_t c_lo = lo == 0 ? 0u
                        : (uint32_t)(((lo - 1) < 4 ? h.z >> (16 * (lo - 1)) : h.w >> (16 * (lo - 5))) & 0xffffull);
                    const uint32_t c_hi =
                        (uint32_t)((hi < 4 ? h.z >> (16 * hi) : h.w >> (16 * (hi - 4))) & 0xffffull);
                    s0 = bstart + c_lo;
                    s1 = bstart + c_hi;
                }
                if (s1 > s0) {
                    first = min(first, s0);
                    last = max(last, s1);
                }
                break;
            }
            if (h0.x == EMPTY_KEY || h1.x == EMPTY_KEY) break;   // end of the chain
            b = next_bucket(b, ht);
        }
    }
    if (first != 0xffffffffu) {
        start = first;
        cnt = last - first;
    }
}

// --------------------------------------------------------------- query prep
// Query keys (grid-stride), validation, and -- for the packed keys-only sort
// -- the digit counts of every pass of its plan (hist != NULL; one pass over
// the keys fewer than a separate histogram kernel).
__global__ void __launch_bounds__(PT, 4) k_qkeys(const double4* __restrict__ Q, uint32_t nq,
                                             GridParams g, unsigned long long* __restrict__ keys,
                                             uint32_t* __restrict__ ids, int shift,
                                             Counters* __restrict__ ctr, const PassPlan plan,
                                             uint32_t* __restrict__ hist) {
    __shared__ uint32_t h[OS_MAXPASS * OS_HSTRIDE];
    if (blockIdx.x == 0 && threadIdx.x == 0) ctr->spill_valid = ~0ull;   // counters zeroed before
    if (hist) {
        for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += PT) h[j] = 0;
        __syncthreads();
    }
    unsigned bad_all = 0;
    auto one = [&](uint32_t i, const double4 s0, const double4 s1) {
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
        bad_all |= bad;
        unsigned long long key = 0;
        if (!bad)
            key = make_key(g, bin_of(g, s0.x), cell_of(g, 0, 0.5 * (s0.y + s1.y)),
                           cell_of(g, 1, 0.5 * (s0.z + s1.z)), cell_of(g, 2, 0.5 * (s0.w + s1.w)));
        if (ids) {
            keys[i] = key;
            ids[i] = i;
        } else {                        // packed: (key, row) in one word, keys-only sort
            const unsigned long long v = (key << shift) | i;
            keys[i] = v;
            if (hist) {
#pragma unroll
                for (int p = 0; p < OS_MAXPASS; ++p)
                    if (p < plan.npass)
                        atomicAdd(&h[p * OS_HSTRIDE + ((v >> plan.shift[p]) & ((1u << plan.bits[p]) - 1u))], 1u);
            }
        }
    };
    // grid-stride, two queries per step with both records' loads issued first
    const uint32_t st = gridDim.x * PT;
    uint32_t i = blockIdx.x * PT + threadIdx.x;
    for (; i < nq && st <= nq - 1 - i; i += 2 * st) {
        const double4 a0 = Q[2 * (size_t)i], a1 = Q[2 * (size_t)i + 1];
        const double4 b0 = Q[2 * (size_t)(i + st)], b1 = Q[2 * (size_t)(i + st) + 1];
        one(i, a0, a1);
        one(i + st, b0, b1);
    }
    if (i < nq) one(i, Q[2 * (size_t)i], Q[2 * (size_t)i + 1]);
    if (bad_all) atomicOr(&ctr->bad, bad_all);
    if (hist) {
        __syncthreads();
        for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += PT)
            if (h[j]) atomicAdd(hist + j, h[j]);
    }
}

// Query order for the grid method ("query segments in Q are sorted by
// non-decreasing t_start"): the top QSB bits of the packed key -- the time
// bin and the top spatial bit on C4 -- in one counting-sort pass.  Each CTA
// takes the exclusive digit bases from k_qkeys' histogram, counts its tile
// in shared memory (the atomics' return values are the ranks), reserves its
// per-digit ranges with one global atomic per digit present, and writes the
// rows.  The order inside a digit is unspecified: it only groups queries
// for locality (results are canonical whatever the order).
constexpr int QS_ITEMS = 8;
__global__ void __launch_bounds__(PT) k_qscatter(const unsigned long long* __restrict__ keys,
                                                uint32_t nq, int shift, int bits,
                                                const uint32_t* __restrict__ hist,
                                                uint32_t* __restrict__ cursor,
                                                unsigned long long row_mask,
                                                uint32_t* __restrict__ order) {
    __shared__ uint32_t base[OS_HSTRIDE], lcnt[OS_HSTRIDE], wsum[PT / 32];
    const uint32_t nd = 1u << bits, t = threadIdx.x, lane = t & 31, warp = t >> 5;
    // the tile's keys and the digit counts are loaded together (one round trip)
    const uint32_t i0 = blockIdx.x * (PT * QS_ITEMS) + t;
    unsigned long long k[QS_ITEMS];
    uint32_t r[QS_ITEMS];
#pragma unroll
    for (int j = 0; j < QS_ITEMS; ++j) {
        const uint32_t i = i0 + (uint32_t)j * PT;
        k[j] = i < nq ? keys[i] : 0ull;
    }
    // exclusive bases of the digits (nd <= 512: two per thread)
    const uint32_t h0 = 2 * t < nd ? hist[2 * t] : 0u, h1 = 2 * t + 1 < nd ? hist[2 * t + 1] : 0u;
    uint32_t inc = h0 + h1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= (uint32_t)o) inc += u;
    }
    if (lane == 31) wsum[warp] = inc;
    lcnt[2 * t] = 0;
    lcnt[2 * t + 1] = 0;
    __syncthreads();
    uint32_t pre = inc - h0 - h1;
    for (uint32_t w = 0; w < warp; ++w) pre += wsum[w];
    base[2 * t] = pre;
    base[2 * t + 1] = pre + h0;
    __syncthreads();
#pragma unroll
    for (int j = 0; j < QS_ITEMS; ++j) {
        const uint32_t i = i0 + (uint32_t)j * PT;
        if (i < nq) r[j] = atomicAdd(&lcnt[(uint32_t)(k[j] >> shift) & (nd - 1u)], 1u);
    }
    __syncthreads();
    for (uint32_t dg = t; dg < nd; dg += PT)
        if (lcnt[dg]) base[dg] += atomicAdd(&cursor[dg], lcnt[dg]);
    __syncthreads();
#pragma unroll
    for (int j = 0; j < QS_ITEMS; ++j) {
        const uint32_t i = i0 + (uint32_t)j * PT;
        if (i < nq) {
            DTS_DCHECK(base[(uint32_t)(k[j] >> shift) & (nd - 1u)] + r[j] < nq);
            order[base[(uint32_t)(k[j] >> shift) & (nd - 1u)] + r[j]] = (uint32_t)(k[j] & row_mask);
        }
    }
}

__global__ void __launch_bounds__(PT) k_unpack_order(const unsigned long long* __restrict__ keys,
                                                    uint32_t n, unsigned long long mask,
                                                    uint32_t* __restrict__ order) {
    const uint32_t i = blockIdx.x * PT + threadIdx.x;
    if (i < n) order[i] = (uint32_t)(keys[i] & mask);
}

// ------------------------------------------------------------- block helpers
#include "wtile.cuh"

// ------------------------------------------------------ re-run bookkeeping
// Tiles re-run after the spill buffer filled: cover[q] = counts[q] for their
// queries (their records in the first spill buffer are stale; the scan of
// cover sizes the re-run's exact spill buffer).
__global__ void __launch_bounds__(PT) k_mark_over(const uint32_t* __restrict__ tiles,
                                                 uint32_t tq,
                                                 const uint32_t* __restrict__ order, uint32_t nq,
                                                 const uint32_t* __restrict__ counts,
                                                 uint32_t* __restrict__ cover) {
    const uint32_t tile = tiles[blockIdx.x];
    const uint32_t sp = tile * tq + threadIdx.x;
    if (threadIdx.x < tq && sp < nq) {
        const uint32_t q = order[sp];
        cover[q] = counts[q];
    }
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

// Per-query candidate counts ("per-query candidate count
// estimate (for balancing)"): the stencil and its row probes exactly as in
// pass 1, summing the run lengths -- the candidates pass 1 will refine --
// without touching a record.  One thread per query; sums per block of
// `block` consecutive queries.
__global__ void __launch_bounds__(PT) k_query_costs(const double4* __restrict__ Q, uint32_t nq,
                                                   double d, GridParams g, HashTable ht,
                                                   const double* __restrict__ bin_t0min,
                                                   const double* __restrict__ bin_t1max,
                                                   const uint32_t* __restrict__ bin_start,
                                                   uint32_t method, SubbinIndex sb,
                                                   uint32_t block, uint32_t stride,
                                                   unsigned long long* __restrict__ out) {
    // thread t evaluates query i = t * stride (its cost counted stride times)
    // (a warp resolving its 32 queries' probes together, as pass 1 does,
    //  measured no faster: 0.045 vs 0.048 ms on C4's 1/8 share, stride 8)
    const uint32_t t = blockIdx.x * PT + threadIdx.x;
    const unsigned long long i64 = (unsigned long long)t * stride;
    const uint32_t i = i64 < nq ? (uint32_t)i64 : nq;
    unsigned long long c = 0;
    if (i < nq) {
        QState q;
        double qlo[3], qhi[3];
        const bool live = load_query(Q, i, q, qlo, qhi);
        const Stencil st = make_stencil(g, q, qlo, qhi, d, live, bin_start, bin_t0min,
                                        bin_t1max, method, sb);
        uint32_t probes = 0;
        for (uint32_t l = 0; l < st.nlook; ++l) {
            uint32_t s0 = 0, cnt = 0;
            resolve(g, ht, bin_t0min, bin_t1max, bin_start, st.mode, st.lb, st.hb, st.clo,
                    st.cn, q.t0, q.t1, l, st.rstart, st.rcnt, s0, cnt, probes);
            c += cnt;
        }
        c *= stride;
    }
    // one atomic per run of lanes with the same output block (a warp's
    // queries share one block unless `block` < 32 x stride or a boundary
    // cuts it)
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t ob = i < nq ? i / block : 0xffffffffu;
    unsigned long long sum = 0;
    uint32_t first = 32;                      // lowest lane of this lane's run
#pragma unroll 4
    for (int k = 0; k < 32; ++k) {
        const unsigned long long v = __shfl_sync(0xffffffffu, c, k);
        const uint32_t ok = __shfl_sync(0xffffffffu, ob, k);
        if (ok == ob) {
            sum += v;
            first = min(first, (uint32_t)k);
        }
    }
    if (ob != 0xffffffffu && lane == first && sum) atomicAdd(&out[ob], sum);
}

// Phase events of one search (time_kernels): sets of six events per thread
// and device, created on first use and recycled in call order (creating
// and destroying them per call cost host time on the call's critical path).
// Mode 2 leaves the elapsed-time reads to dts_search_read_times, after the
// caller's timed region.
constexpr uint32_t TIMER_SETS = 1024;
struct TimerRing {
    cudaEvent_t ev[TIMER_SETS][6];
    bool made[TIMER_SETS] = {false};
    uint32_t next = 0;            // calls so far (slot = next % TIMER_SETS)
    uint32_t rec[TIMER_SETS] = {0};   // bit j: event j (phase boundary j) recorded
};
TimerRing& timer_ring(int dev) {
    static thread_local TimerRing* rings[64] = {nullptr};
    if (dev < 0 || dev >= 64) throw Error(DTS_ENOTSUP, "device ordinal >= 64");
    if (!rings[dev]) rings[dev] = new TimerRing();
    return *rings[dev];
}

// mode 1, 2: all six phase boundaries; mode 3: only pass 1's two (a timing
// event between two kernels costs the stream a few microseconds: six of them
// add ~25 us to a C4 search, two ~8)
struct EventTimer {
    bool on;
    cudaStream_t s;
    cudaEvent_t* ev = nullptr;
    uint32_t* rec = nullptr;
    uint32_t want = 0x3f, rec0 = 0;
    int calls = 0;
    uint32_t handle = 0;
    EventTimer(uint32_t mode, cudaStream_t st) : on(mode != 0), s(st) {
        rec = &rec0;
        if (!on) return;
        if (mode == 3) want = (1u << 1) | (1u << 2);
        int dev = 0;
        DTS_CUDA(cudaGetDevice(&dev));
        TimerRing& r = timer_ring(dev);
        handle = r.next++;
        const uint32_t i = handle % TIMER_SETS;
        if (!r.made[i]) {
            for (auto& e : r.ev[i]) DTS_CUDA(cudaEventCreate(&e));
            r.made[i] = true;
        }
        ev = r.ev[i];
        rec = &r.rec[i];
        *rec = 0;
    }
    void mark() {
        if (on && calls < 6 && ((want >> calls) & 1u)) {
            DTS_CUDA(cudaEventRecord(ev[calls], s));
            *rec |= 1u << calls;
        }
        ++calls;
    }
    float ms(int i) {
        float t = 0.f;
        if (on && ((*rec >> i) & 3u) == 3u) cudaEventElapsedTime(&t, ev[i], ev[i + 1]);
        return t;
    }
};

}  // namespace

void search_device(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                   uint32_t qid_base, cudaStream_t s, SearchOut* out, dts_search_stats* stats,
                   unsigned long long max_results, const uint32_t* qmap,
                   const uint32_t* qtraj, bool exclude_same_traj, bool count_only,
                   uint32_t* counts_out) {
    out->results = nullptr;
    HostTrace tr("search");
    out->count = 0;
    dts_search_stats local{};
    if (stats) local.time_kernels = stats->time_kernels;
    local.timer_slot = 0xffffffffu;               // set when phase events are recorded
    if (nq == 0) {
        if (stats) *stats = local;
        return;
    }
    if (idx->ooc) {              // D in temporal shards on the host (ooc.cu)
        ooc_search(idx, Q_dev, nq, d, qid_base, s, out, stats, qmap, qtraj, exclude_same_traj,
                   count_only, counts_out);
        return;
    }
    const double4* Q = reinterpret_cast<const double4*>(Q_dev);
    // the counters and the query sort's digit counts in one buffer, zeroed by
    // one memset (spill_valid is set to ~0 by k_qkeys)
    constexpr size_t CTR_BYTES = (sizeof(Counters) + 255) / 256 * 256;
    constexpr size_t HIST_N = (size_t)OS_MAXPASS * OS_HSTRIDE;
    DevBuf<unsigned char> small(CTR_BYTES + HIST_N * sizeof(uint32_t), s);
    Counters* const ctr_p = reinterpret_cast<Counters*>(small.p);
    uint32_t* const hist_p = reinterpret_cast<uint32_t*>(small.p + CTR_BYTES);
    DTS_CUDA(cudaMemsetAsync(small.p, 0, small.n, s));
    tr.mark("ctr");

    if (idx->n == 0) {   // empty index: validate only
        k_validate_only<<<blocks(nq, PT), PT, 0, s>>>(Q, (uint32_t)nq, ctr_p);
        DTS_LAUNCH_CHECK();
        Counters hc;
        DTS_CUDA(cudaMemcpyAsync(&hc, ctr_p, sizeof(hc), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        if (hc.bad) throw Error(DTS_EINVAL, "invalid query segment (non-finite or t_end < t_start)");
        if (count_only && counts_out) {
            DTS_CUDA(cudaMemsetAsync(counts_out, 0, nq * sizeof(uint32_t), s));
            DTS_CUDA(cudaStreamSynchronize(s));
        }
        if (stats) *stats = local;
        return;
    }

    EventTimer tm(local.time_kernels, s);
    tm.mark();
    static const int nsm_prep = [] {
        int dev = 0, v = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
        return v;
    }();
    // expected candidates per query: entries per non-empty cell x stencil
    // cells x bins a query spans (sizes the query sort and the warp tiles)
    double work = idx->n_cells ? (double)idx->n / (double)idx->n_cells : 0.0;
    for (int a = 0; a < 3; ++a)
        work *= std::floor(2.0 * (d + idx->gp.half_ext[a]) / idx->gp.w[a]) + 2.0;
    work *= std::floor(idx->gp.maxdur / idx->gp.b) + 2.0;
    // ---- query prep: key + sort
    // query keys (and the multi-pass sort's second key buffer) and the order
    // in one allocation
    DevBuf<unsigned char> prepbuf(nq * (2 * sizeof(unsigned long long) + sizeof(uint32_t)), s);
    uint32_t* const order_p =
        reinterpret_cast<uint32_t*>(prepbuf.p + nq * 2 * sizeof(unsigned long long));
    {
        // packed (key << row bits | row) keys-only sort when it fits 64 bits
        const int row_bits = std::max(1, bits_for(nq - 1));
        const bool packed = row_bits + idx->key_bits <= 64;
        // below DTS_QSORT_MIN queries (default 2^18) the sort -- about ten
        // small launches -- costs more than the locality it buys, and the
        // queries keep their order.  Device search time, sorted -> unsorted:
        // C1 (10 k queries) 0.166 -> 0.107 ms, C2 (100 k) 0.338 -> 0.233,
        // C3 (100 k) 0.481 -> 0.406, S2 (51 k) 7.27 -> 6.63, S3 (51 k)
        // 0.231 -> 0.143; S1 (40 k) 3.38 -> 3.61
        static const size_t qsort_min = [] {
            const char* e = getenv("DTS_QSORT_MIN");
            return e ? (size_t)atoll(e) : ((size_t)1 << 18);
        }();
        // (the temporal and subbin methods always sort: their one-run queries
        // are grouped by identical run inside a tile, which needs neighbours)
        // ... and output-heavy grid searches sort too: expected candidates
        // per query (entries per non-empty cell x stencil cells) over
        // DTS_QSORT_WORK (default 1024): neighbouring queries then share
        // their rows in L1/L2 (C2 at d = 8, 100 k queries: pass 1 3.72 ->
        // 3.11 ms sorted; at d = 2, ~40 candidates per query, sorting costs
        // more than it saves)
        static const double qsort_work = [] {
            const char* e = getenv("DTS_QSORT_WORK");
            return e ? atof(e) : 1024.0;
        }();
        const bool sort_q = nq >= qsort_min || idx->method != DTS_METHOD_GRID ||
                            (idx->method == DTS_METHOD_GRID && work >= qsort_work);
        static const int drop = [] {           // DTS_QSORT_DROP: low key bits left unsorted
            const char* e = getenv("DTS_QSORT_DROP");
            return e ? std::max(0, std::min(24, atoi(e))) : -1;
        }();
        // the order only serves locality: by default only the key's top 16
        // bits (bin and the slowest cell axis) are sorted, two radix passes
        // (C4, 34-bit keys: all but key_bits % 8 = 2 bits, four passes: prep
        // 0.122 ms, pass 1 0.618; top 24 bits: 0.104, 0.616; top 16: 0.084,
        // 0.617).  The packed sort's digit counts come from k_qkeys and its
        // last pass writes the order itself.
        // grid method: the top 9 key bits (the bin) in one counting
        // pass (k_qscatter; DTS_QSORT_DROP selects the multi-pass sort);
        // C4: pass 1 0.577 -> 0.565 ms (queries of one bin
        // in their given order load the memory system more evenly than
        // cell-sorted ones)
        const bool one_pass = sort_q && packed && drop < 0 && idx->method == DTS_METHOD_GRID &&
                              nq > 1 && idx->key_bits > 0;
        const int dr = drop >= 0 ? drop : std::max(0, idx->key_bits - 16);
        const int lo = one_pass ? row_bits + std::max(0, idx->key_bits - 9)
                                : row_bits + std::min(dr, std::max(0, idx->key_bits - 8));
        const bool fused = !one_pass && sort_q && packed && radix_onesweep(nq) && nq > 1 &&
                           row_bits + idx->key_bits > lo;
        const PassPlan plan = fused ? plan_passes(lo, row_bits + idx->key_bits, true)
                                    : (one_pass ? PassPlan{1, {lo}, {row_bits + idx->key_bits - lo}}
                                                : PassPlan{});
        unsigned long long* const qk_p = reinterpret_cast<unsigned long long*>(prepbuf.p);
        unsigned long long* const qk_tmp_p = qk_p + nq;
        // (hist_p: the digit counts, zeroed with the counters; one_pass: the
        //  digit counts, then the per-digit cursors)
        k_qkeys<<<(unsigned)std::min<size_t>(blocks(nq, PT), (size_t)nsm_prep * 4), PT, 0, s>>>(
            Q, (uint32_t)nq, idx->gp, qk_p, (packed && sort_q) ? nullptr : order_p, row_bits,
            ctr_p, plan, (fused || one_pass) ? hist_p : nullptr);
        DTS_LAUNCH_CHECK();
        if (one_pass) {
            k_qscatter<<<blocks(nq, PT * QS_ITEMS), PT, 0, s>>>(
                qk_p, (uint32_t)nq, plan.shift[0], plan.bits[0], hist_p, hist_p + OS_HSTRIDE,
                (1ull << row_bits) - 1ull, order_p);
            DTS_LAUNCH_CHECK();
        } else if (!sort_q) {
            // order = identity (written by k_qkeys)
        } else if (fused) {
            radix_sort_keys_hist(qk_p, qk_tmp_p, nq, plan, hist_p, s, order_p,
                                 (1ull << row_bits) - 1ull);
        } else if (packed) {
            const unsigned long long* sorted =
                radix_sort_keys(qk_p, qk_tmp_p, nq, lo, row_bits + idx->key_bits, s);
            k_unpack_order<<<blocks(nq, PT), PT, 0, s>>>(sorted, (uint32_t)nq,
                                                        (1ull << row_bits) - 1ull, order_p);
            DTS_LAUNCH_CHECK();
        } else {
            DevBuf<uint32_t> order_tmp(nq, s);
            radix_sort_pairs(qk_p, order_p, qk_tmp_p, order_tmp.p, nq, idx->key_bits, s);
        }
    }
    // the build may still run (dts_build_index_device returns once its last
    // kernels are enqueued): the query prep above needs only the grid
    // parameters, so on another stream it overlaps the build's tail; pass 1
    // reads the index and waits for it here (inside the prep phase's events,
    // so ms_count times pass 1 alone)
    if (idx->ready) DTS_CUDA(cudaStreamWaitEvent(s, idx->ready, 0));
    tm.mark();
    tr.mark("prep");

    // ---- pass 1: warp tiles, count + staging (spilling output-heavy tiles)
    // queries per warp tile: WQ, or fewer when the query set would not give
    // every resident warp of pass 1 F tiles -- a small set then runs on more
    // warps, each with a shorter latency chain -- with F = 2.5 and at least 4
    // queries; heavy queries (work >= 160 expected candidates, about 40
    // actual: the estimate runs ~4x high) F = 12 and at least 2; work >=
    // 4000: F = 24, tiles down to one query.  Measured
    // (device search, ms, tiles of 2 / 4 / 7 / 10 / 16 queries): C1 0.146 /
    // 0.131 / 0.131 / 0.134 / 0.143; C2 d = 2 0.377 / 0.382 / 0.389 / 0.432 /
    // 0.466; C2 d = 8 3.42 / 3.45 / 3.61 / 3.76 / 4.15; S1 d = 50 0.201 /
    // 0.189 / 0.229 / 0.220 / 0.250; S2 d = 0.1 0.643 / 0.744 / 0.899 /
    // 0.979 / 1.329; S3 d = 0.01 0.215 / 0.181 / 0.169 / 0.174 / 0.166; the
    // C4 query set's 1/8 (125 k, a rank's share at N = 8): 8 0.209, 13 0.184,
    // 16 0.187.  F: 2 / 2.5 / 4 -- S1 d = 50 0.204 / 0.168 / 0.168, S3 d =
    // 0.05 0.157 / 0.167 / 0.167, the C4 1/8 share 0.185 / 0.184 / 0.209.
    // Heavy (tiles of 1 / 2 / 3 / 4): S2 d = 1 29.3 / 31.0 / 32.6 / 34.0;
    // S2 d = 0.1 0.632 / 0.625 / 0.678 / 0.720; C2 d = 8 3.42 / 3.40 / 3.40 /
    // 3.43; C2 d = 2 0.597 / 0.360 / - / 0.382
    static const int nsm_tiles = [] {
        int dev = 0, v = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
        return v;
    }();
    static const double tile_fill = [] {        // DTS_TILE_FILL: F for light queries
        const char* e = getenv("DTS_TILE_FILL");  // (0: always WQ)
        return e ? atof(e) : 2.5;
    }();
    const double slots = (double)nsm_tiles * 7.0 * WW;            // resident warps of pass 1
    const double fill = work >= 4000.0 ? 9.6 * tile_fill : (work >= 160.0 ? 4.8 * tile_fill : tile_fill);
    const double tmin = work >= 4000.0 ? 1.0 : (work >= 160.0 ? 2.0 : 4.0);
    // (the temporal and subbin methods keep WQ: their tiles' queries share
    //  runs, streamed once per group)
    uint32_t tq = (tile_fill <= 0.0 || idx->method != DTS_METHOD_GRID) ? (uint32_t)WQ
        : (uint32_t)std::max(tmin, std::min((double)WQ, std::ceil((double)nq / (fill * slots))));
    static const int tile_q_env = [] {          // DTS_TILE_Q: a fixed tile size (A/B)
        const char* e = getenv("DTS_TILE_Q");
        return e ? std::max(1, std::min(WQ, atoi(e))) : 0;
    }();
    if (tile_q_env && idx->method == DTS_METHOD_GRID) tq = (uint32_t)tile_q_env;
    const uint32_t ntiles = (uint32_t)((nq + tq - 1) / tq);
    // (DTS_STAGE_CAP: a fixed staging capacity, testing knob for the re-run
    //  of tiles that find the stage full)
    static const long long stage_env = [] {
        const char* e = getenv("DTS_STAGE_CAP");
        return e ? atoll(e) : -1ll;
    }();
    unsigned long long stage_cap = stage_env >= 0 ? (unsigned long long)stage_env
                                                  : 4ull * nq + (1ull << 20);
    // spill buffer: sized from the largest output this index has seen (a
    // repeated output-heavy search spills without re-runs), at least 8
    // records per query
    // (DTS_SPILL_CAP: a fixed capacity, testing knob for the re-run path)
    static const long long spill_env = [] {
        const char* e = getenv("DTS_SPILL_CAP");
        return e ? atoll(e) : -1ll;
    }();
    unsigned long long spill_cap = spill_env >= 0 ? (unsigned long long)spill_env
        : std::max<unsigned long long>(8ull * nq + (1ull << 20),
                                       idx->spill_hint.load(std::memory_order_relaxed));
    // pass-1 bookkeeping in one allocation (256-byte aligned pieces)
    size_t p1_bytes = 0;
    auto piece = [&](size_t bytes) {
        const size_t o = p1_bytes;
        p1_bytes += (bytes + 255) / 256 * 256;
        return o;
    };
    const size_t o_counts = piece(nq * 4), o_over = piece((size_t)ntiles * 4),
                 o_stiles = piece((size_t)ntiles * 4), o_off = piece((nq + 1) * 8),
                 o_tbase = piece((size_t)ntiles * 8), o_qstage = piece(count_only ? 0 : nq * 8);
    DevBuf<unsigned char> p1buf(p1_bytes, s);
    uint32_t* const counts_p = reinterpret_cast<uint32_t*>(p1buf.p + o_counts);
    uint32_t* const over_tiles_p = reinterpret_cast<uint32_t*>(p1buf.p + o_over);
    uint32_t* const spill_tiles_p = reinterpret_cast<uint32_t*>(p1buf.p + o_stiles);
    unsigned long long* const offsets_p = reinterpret_cast<unsigned long long*>(p1buf.p + o_off);
    unsigned long long* const tile_base_p = reinterpret_cast<unsigned long long*>(p1buf.p + o_tbase);
    unsigned long long* const qstage_p =
        count_only ? nullptr : reinterpret_cast<unsigned long long*>(p1buf.p + o_qstage);
    DevBuf<dts_result> stage(stage_cap, s);
    DevBuf<uint2> spill(std::max<unsigned long long>(spill_cap, 1), s);        // (query, entry)
    DevBuf<double2> spill_t(std::max<unsigned long long>(spill_cap, 1), s);    // intervals
    tr.mark("bufs");
    TileArgs ta{};
    ta.Q = Q;
    ta.order = order_p;
    ta.nq = (uint32_t)nq;
    ta.d = d;
    ta.g = idx->gp;
    ta.soa = idx->soa;
    ta.ht = idx->ht;
    ta.bin_t0min = idx->bin_t0min;
    ta.bin_t1max = idx->bin_t1max;
    ta.bin_start = idx->bin_start;
    ta.counts = counts_p;
    ta.stage = stage.p;
    ta.stage_cap = stage_cap;
    ta.tile_base = tile_base_p;
    ta.over_tiles = over_tiles_p;
    ta.spill_tiles = spill_tiles_p;
    ta.spill_qe = spill.p;
    ta.spill_t = spill_t.p;
    ta.spill_cap = spill_cap;
    ta.tile_list = nullptr;
    ta.n_list = 0;
    ta.spill_all = 0;
    ta.count_only = count_only ? 1u : 0u;
    ta.qid_base = qid_base;
    ta.qmap = qmap;
    ta.etraj = idx->etraj;
    ta.qtraj = qtraj;
    ta.excl = (qtraj && idx->etraj && exclude_same_traj) ? 1u : 0u;
    if (exclude_same_traj && !(qtraj && idx->etraj))
        throw Error(DTS_EINVAL, "exclude_same_trajectory needs query_traj and an index built "
                                "with entry_traj");
    ta.ctr = ctr_p;
    ta.method = idx->method;
    ta.sb = idx->sb;
    ta.out = idx->out;
    ta.qstage = count_only ? nullptr : qstage_p;
    ta.tq = tq;
    local.tile_queries = tq;
    local.work_estimate = (float)work;
    int nsm = 148;
    {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    }
    // CTAs per SM the grid kernel is register-bounded for (DTS_TILE_OCC =
    // 6..8: 85, 73 or 64 registers per thread; measured on C4 (one box, 20
    // steps): 6: 1.00 ms, 7: 0.86, 8: 0.92)
    static const int occ = [] {
        const char* e = getenv("DTS_TILE_OCC");
        const int v = e ? atoi(e) : 7;
        return (v == 5 || v == 6 || v == 8) ? v : 7;
    }();
    auto launch_pass1 = [&](const TileArgs& args, uint32_t tiles) {
        const unsigned want = (tiles + WW - 1) / WW;
        const unsigned g7 = std::min<unsigned>(want, nsm * 7);
        if (args.out.okeys) {             // the index holds long-segment copies
            if (args.count_only) {
                if (args.excl) k_wtile_count<7, false, false, true, true, true><<<g7, WT, 0, s>>>(args);
                else k_wtile_count<7, false, false, false, true, true><<<g7, WT, 0, s>>>(args);
            } else if (args.excl) {
                k_wtile_count<7, false, false, true, true><<<g7, WT, 0, s>>>(args);
            } else {
                k_wtile_count<7, false, false, false, true><<<g7, WT, 0, s>>>(args);
            }
        } else if (args.excl) {           // exclude_same_trajectory instantiations
            if (idx->method == DTS_METHOD_SUBBIN) k_wtile_count<7, true, true, true><<<g7, WT, 0, s>>>(args);
            else if (idx->method == DTS_METHOD_TEMPORAL) k_wtile_count<7, false, true, true><<<g7, WT, 0, s>>>(args);
            else k_wtile_count<7, false, false, true><<<g7, WT, 0, s>>>(args);
        } else if (idx->method == DTS_METHOD_SUBBIN) {
            k_wtile_count<7, true, true><<<g7, WT, 0, s>>>(args);
        } else if (idx->method == DTS_METHOD_TEMPORAL) {
            k_wtile_count<7, false, true><<<g7, WT, 0, s>>>(args);
        } else if (occ == 8) {
            k_wtile_count<8><<<std::min<unsigned>(want, nsm * 8), WT, 0, s>>>(args);
        } else if (occ == 5) {
            k_wtile_count<5><<<std::min<unsigned>(want, nsm * 5), WT, 0, s>>>(args);
        } else if (occ == 6) {
            k_wtile_count<6><<<std::min<unsigned>(want, nsm * 6), WT, 0, s>>>(args);
        } else {
            k_wtile_count<7><<<g7, WT, 0, s>>>(args);
        }
        DTS_LAUNCH_CHECK();
    };
    launch_pass1(ta, ntiles);
    tr.mark("pass1");
    if (ta.out.okeys && !count_only) {
        // ---- long-segment copies: spilled records carry sorted positions
        //      and their tiles' counts include hits on non-canonical copies;
        //      both are fixed before the scan (k_spill_filter).  A tile that
        //      overflowed a buffer (counts unfiltered, or hits not kept)
        //      sends pass 1 round again, the overflowed buffer sized by the
        //      sum of the counts (an upper bound of what it must hold).
        Counters c1;
        DTS_CUDA(cudaMemcpyAsync(&c1, ctr_p, sizeof(c1), cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        if (c1.n_over) {
            scan_exclusive_u32_to_u64(counts_p, offsets_p, nq, s);
            unsigned long long bound = 0;
            DTS_CUDA(cudaMemcpyAsync(&bound, offsets_p + nq, sizeof(bound),
                                     cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaStreamSynchronize(s));
            if (c1.staged > stage_cap) {
                stage_cap = std::max(stage_cap, bound);
                stage.alloc(stage_cap, s);
                ta.stage = stage.p;
                ta.stage_cap = stage_cap;
            }
            if (c1.spill_valid != ~0ull) {
                spill_cap = std::max(spill_cap, bound);
                spill.alloc(std::max<unsigned long long>(spill_cap, 1), s);
                spill_t.alloc(std::max<unsigned long long>(spill_cap, 1), s);
                ta.spill_qe = spill.p;
                ta.spill_t = spill_t.p;
                ta.spill_cap = spill_cap;
                unsigned long long want = bound + (1ull << 20), cur = idx->spill_hint.load();
                while (cur < want && !idx->spill_hint.compare_exchange_weak(cur, want)) {}
            }
            DTS_CUDA(cudaMemsetAsync(ctr_p, 0, sizeof(Counters), s));
            DTS_CUDA(cudaMemsetAsync(&ctr_p->spill_valid, 0xFF, sizeof(unsigned long long), s));
            launch_pass1(ta, ntiles);
            DTS_CUDA(cudaMemcpyAsync(&c1, ctr_p, sizeof(c1), cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaStreamSynchronize(s));
            if (c1.n_over) throw Error(DTS_EINTERNAL, "pass 1 overflowed buffers sized by its counts");
        }
        const unsigned long long n1 = std::min(c1.spilled, spill_cap);
        if (n1) {
            k_spill_filter<<<(unsigned)std::min<unsigned long long>(blocks(n1, 128), nsm * 8ull), 128,
                             0, s>>>(ta, n1, spill.p);
            DTS_LAUNCH_CHECK();
        }
        if (c1.n_spill) {
            k_spill_max<<<blocks((size_t)c1.n_spill * tq, 128), 128, 0, s>>>(
                spill_tiles_p, c1.n_spill, tq, order_p, (uint32_t)nq, counts_p, ctr_p);
            DTS_LAUNCH_CHECK();
        }
    }
    tm.mark();
    scan_exclusive_u32_to_u64(counts_p, offsets_p, nq, s, &ctr_p->total);
    tm.mark();
    tr.mark("scan");

    // pass 2: staged hits gathered into the output
    auto launch_emit = [&](dts_result* dst, unsigned long long cap) {
        k_emit_gather<<<(unsigned)blocks(nq, 256), 256, 0, s>>>(
            (uint32_t)nq, counts_p, offsets_p, qstage_p, stage.p, stage_cap, dst, cap);
    };
    // pass 2 launched before the host learns the total, into a buffer sized
    // by this index's previous result count: a repeated search of one index
    // then has no host round trip between the scan and the copy (a buffer
    // that turns out too small is freed and pass 2 launched again)
    struct SpecOut {
        dts_result* p = nullptr;
        cudaStream_t s = nullptr;
        ~SpecOut() {
            if (p) {
                cudaStreamSynchronize(s);
                cache_free(p);
            }
        }
    } spec;
    spec.s = s;
    // (the hint scales the last search's results per query to this query
    //  set: chunks of one host search differ in size)
    const double rate = count_only ? 0.0 : idx->result_hint.load();
    const unsigned long long hint =
        rate > 0.0 ? (unsigned long long)(rate * (double)nq * 1.125) + 4096ull : 0ull;
    static const bool spec_on = [] {          // DTS_SPEC_EMIT=0: off
        const char* e = getenv("DTS_SPEC_EMIT");
        return !(e && e[0] == '0');
    }();
    if (spec_on && hint > 0) {
        spec.p = static_cast<dts_result*>(cache_alloc(hint * sizeof(dts_result)));
        launch_emit(spec.p, hint);
        DTS_LAUNCH_CHECK();
    }
    // counters and total read back through a pinned buffer of the calling
    // thread (a pageable destination adds a staging copy to the call)
    struct Readback {
        Counters c;
        unsigned long long total;
    };
    struct RbHolder {
        Readback* p = nullptr;
        ~RbHolder() { if (p) cudaFreeHost(p); }   // thread exit (stream workers)
    };
    static thread_local RbHolder rbh;
    if (!rbh.p) DTS_CUDA(cudaMallocHost((void**)&rbh.p, sizeof(Readback)));
    Readback* rb = rbh.p;
    DTS_CUDA(cudaMemcpyAsync(&rb->c, ctr_p, sizeof(Counters), cudaMemcpyDeviceToHost, s));
    tr.mark("emit");
    DTS_CUDA(cudaStreamSynchronize(s));
    tr.mark("sync");
    Readback h = *rb;
    h.total = h.c.total;
    if (!count_only) idx->result_hint.store((double)h.total / (double)nq);
    if (h.c.bad & 1) throw Error(DTS_EINVAL, "query segment with a non-finite coordinate or time");
    if (h.c.bad & 2) throw Error(DTS_EINVAL, "query segment with t_end < t_start");
    if (h.c.bad & 4) throw Error(DTS_EINVAL, "query segment whose speed overflows fp64");
    local.candidates = h.c.candidates;
    local.cell_lookups = h.c.lookups;
    local.results = h.total;
    local.max_results_per_query = h.c.max_count;
    if (count_only) {                   // counts and total only (dts_search_count)
        if (counts_out && nq)
            DTS_CUDA(cudaMemcpyAsync(counts_out, counts_p, nq * sizeof(uint32_t),
                                     cudaMemcpyDefault, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        out->count = (size_t)h.total;
        tm.mark();
        tm.mark();
        if (local.time_kernels >= 2) {
            local.timer_slot = tm.handle;
        } else if (local.time_kernels) {
            local.ms_prep = tm.ms(0);
            local.ms_count = tm.ms(1);
            local.ms_scan = tm.ms(2);
        }
        if (stats) *stats = local;
        return;
    }
    if (h.c.n_over) {
        // the spill buffer filled: size the next search's from this output
        unsigned long long want = h.total + (1ull << 20), cur = idx->spill_hint.load();
        while (cur < want && !idx->spill_hint.compare_exchange_weak(cur, want)) {}
    }

    // ---- results that do not fit the device: report the per-query counts
    //      so a host caller can stream the search in query chunks
    const double per = h.c.n_over ? 24.0 + 24.0 : 24.0;   // fin (+ the re-run's spill)
    // (cudaMemGetInfo is slow and jittery -- up to 15 ms measured on S2 at
    //  d = 1 with 30 GB of pool memory mapped -- so it is asked only when the
    //  results could take more than a quarter of the device's memory)
    static const double dev_bytes = [] {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceProp pr;
        return cudaGetDeviceProperties(&pr, dev) == cudaSuccess ? (double)pr.totalGlobalMem : 0.0;
    }();
    if (h.total > 0 && ((double)h.total * per > 0.25 * dev_bytes || h.total > max_results)) {
        size_t free_b = 0, total_b = 0;
        DTS_CUDA(cudaMemGetInfo(&free_b, &total_b));
        if ((double)h.total * per > 0.8 * (double)free_b || h.total > max_results) {
            ResultsTooLarge e(h.total);
            e.counts.resize(nq);
            DTS_CUDA(cudaMemcpyAsync(e.counts.data(), counts_p, nq * sizeof(uint32_t),
                                     cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaStreamSynchronize(s));
            throw e;
        }
    }

    if (h.total > 0) {
        dts_result* fin = nullptr;
        bool emitted = false;
        if (spec.p && h.total <= hint) {        // the speculative pass 2 holds it all
            fin = spec.p;
            spec.p = nullptr;
            emitted = true;
        } else {
            if (spec.p) {
                DTS_CUDA(cudaStreamSynchronize(s));
                cache_free(spec.p);
                spec.p = nullptr;
            }
            fin = static_cast<dts_result*>(cache_alloc(h.total * sizeof(dts_result)));
        }
        try {
            // ---- pass 2: staged tiles are copied to their exact offsets
            if (!emitted) {
                launch_emit(fin, h.total);
                DTS_LAUNCH_CHECK();
            }
            tm.mark();
            if (h.c.n_spill || h.c.n_over) {
                DevBuf<uint32_t> cursor(nq, s), cover(h.c.n_over ? nq : 0, s);
                DTS_CUDA(cudaMemsetAsync(cursor.p, 0, nq * sizeof(uint32_t), s));
                DevBuf<uint2> spill2(0, s);
                DevBuf<double2> spill2_t(0, s);
                unsigned long long n_raw = 0;
                if (h.c.n_over) {
                    // ---- tiles that found the spill buffer full: pass 1
                    //      again over those tiles only, every hit spilled
                    //      into a buffer of exactly their result count
                    DevBuf<unsigned long long> cover_off(nq + 1, s);
                    DTS_CUDA(cudaMemsetAsync(cover.p, 0, nq * sizeof(uint32_t), s));
                    k_mark_over<<<h.c.n_over, PT, 0, s>>>(over_tiles_p, tq, order_p, (uint32_t)nq,
                                                          counts_p, cover.p);
                    DTS_LAUNCH_CHECK();
                    scan_exclusive_u32_to_u64(cover.p, cover_off.p, nq, s);
                    DTS_CUDA(cudaMemcpyAsync(&n_raw, cover_off.p + nq, sizeof(n_raw),
                                             cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                    spill2.alloc(std::max<unsigned long long>(n_raw, 1), s);
                    spill2_t.alloc(std::max<unsigned long long>(n_raw, 1), s);
                    DevBuf<Counters> ctr2(1, s);
                    DTS_CUDA(cudaMemsetAsync(ctr2.p, 0, sizeof(Counters), s));
                    DTS_CUDA(cudaMemsetAsync(&ctr2.p->spill_valid, 0xFF, 8, s));
                    TileArgs tb = ta;
                    tb.ctr = ctr2.p;
                    tb.spill_qe = spill2.p;
                    tb.spill_t = spill2_t.p;
                    tb.spill_cap = n_raw;
                    tb.tile_list = over_tiles_p;
                    tb.n_list = h.c.n_over;
                    tb.spill_all = 1;
                    launch_pass1(tb, h.c.n_over);
                }
                // ---- spilled records to their query segments of a scratch
                //      mirror of the output, then each segment sorted by
                //      entry id into the output
                // keys (entry id << 32 | spill index) placed by query, then
                // sorted; the records gathered from the spill buffers
                DevBuf<unsigned long long> rkeys(h.total, s);
                const unsigned long long n1 = std::min(std::min(h.c.spilled, spill_cap),
                                                       h.c.spill_valid);
                if (n1 + n_raw >= (1ull << 32))
                    throw Error(DTS_ENOTSUP, "more than 2^32 spilled results in one search call");
                const SpillSrc src{spill_t.p, n1, spill2_t.p};
                if (n1) {
                    k_spill_place<<<blocks(n1, 256), 256, 0, s>>>(
                        spill.p, n1, 0u, h.c.n_over ? cover.p : nullptr, offsets_p, cursor.p,
                        rkeys.p);
                    DTS_LAUNCH_CHECK();
                }
                if (n_raw) {
                    k_spill_place<<<blocks(n_raw, 256), 256, 0, s>>>(
                        spill2.p, n_raw, (uint32_t)n1, nullptr, offsets_p, cursor.p, rkeys.p);
                    DTS_LAUNCH_CHECK();
                }
                DevBuf<uint32_t> bigc(nq, s);
                DTS_CUDA(cudaMemsetAsync(bigc.p, 0, nq * sizeof(uint32_t), s));
                DTS_CUDA(cudaMemsetAsync(&ctr_p->n_big, 0, 5 * sizeof(unsigned int), s));
                const size_t nslots = ((size_t)h.c.n_spill + h.c.n_over) * tq;
                DevBuf<uint32_t> lists(4 * nslots, s);       // 3 size classes + long segments
                const int eb = idx->eid_bits;
                if (h.c.n_spill) {
                    k_seg_sort_warp<<<blocks((size_t)h.c.n_spill * tq, 4), 128, 0, s>>>(
                        spill_tiles_p, h.c.n_spill * tq, tq, order_p, (uint32_t)nq, counts_p,
                        offsets_p, rkeys.p, src, qmap, qid_base, eb, fin, lists.p, nslots, bigc.p,
                        ctr_p);
                    DTS_LAUNCH_CHECK();
                }
                if (h.c.n_over) {
                    k_seg_sort_warp<<<blocks((size_t)h.c.n_over * tq, 4), 128, 0, s>>>(
                        over_tiles_p, h.c.n_over * tq, tq, order_p, (uint32_t)nq, counts_p,
                        offsets_p, rkeys.p, src, qmap, qid_base, eb, fin, lists.p, nslots, bigc.p,
                        ctr_p);
                    DTS_LAUNCH_CHECK();
                }
                unsigned int nbm[5] = {0, 0, 0, 0, 0};   // n_big, n_cls[3], n_skew
                DTS_CUDA(cudaMemcpyAsync(nbm, &ctr_p->n_big, sizeof(nbm),
                                         cudaMemcpyDeviceToHost, s));
                DTS_CUDA(cudaStreamSynchronize(s));
                static const bool smem_ok = [] {
                    return cudaFuncSetAttribute(k_seg_radix<1024, 16, 1>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_CAP * 8) == cudaSuccess &&
                           cudaFuncSetAttribute(k_seg_bucket<1024, 16, 1>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_CAP * 12) == cudaSuccess &&
                           cudaFuncSetAttribute(k_seg_bucket<512, 16, 2>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_MID2 * 12) == cudaSuccess &&
                           cudaFuncSetAttribute(k_seg_bucket<512, 8, 2>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_MID * 12) == cudaSuccess &&
                           cudaFuncSetAttribute(k_seg_bucket<1024, 16, 1, true>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_CAP * 12) == cudaSuccess &&
                           cudaFuncSetAttribute(k_seg_radix<1024, 16, 1, true>,
                                                cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                SEG_CAP * 8) == cudaSuccess;
                }();
                if (!smem_ok) throw Error(DTS_ECUDA, "segment sort: shared memory size refused");
                DevBuf<uint32_t> skew_list(nbm[1] + nbm[2] + nbm[3], s);
                if (nbm[1]) {
                    k_seg_bucket<512, 8, 2><<<nbm[1], 512, SEG_MID * 12, s>>>(
                        lists.p, counts_p, offsets_p, rkeys.p, src, qmap, qid_base, fin,
                        skew_list.p, ctr_p, SegDesc{});
                    DTS_LAUNCH_CHECK();
                }
                if (nbm[2]) {
                    k_seg_bucket<512, 16, 2><<<nbm[2], 512, SEG_MID2 * 12, s>>>(
                        lists.p + nslots, counts_p, offsets_p, rkeys.p, src, qmap, qid_base, fin,
                        skew_list.p, ctr_p, SegDesc{});
                    DTS_LAUNCH_CHECK();
                }
                if (nbm[3]) {
                    k_seg_bucket<1024, 16, 1><<<nbm[3], 1024, SEG_CAP * 12, s>>>(
                        lists.p + 2 * nslots, counts_p, offsets_p, rkeys.p, src, qmap, qid_base,
                        fin, skew_list.p, ctr_p, SegDesc{});
                    DTS_LAUNCH_CHECK();
                }
                unsigned int n_skew = 0;
                if (nbm[1] + nbm[2] + nbm[3]) {
                    DTS_CUDA(cudaMemcpyAsync(&n_skew, &ctr_p->n_skew, sizeof(n_skew),
                                             cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                }
                if (n_skew) {
                    k_seg_radix<1024, 16, 1><<<n_skew, 1024, SEG_CAP * 8, s>>>(
                        skew_list.p, counts_p, offsets_p, rkeys.p, src, qmap, qid_base, eb, fin,
                        SegDesc{});
                    DTS_LAUNCH_CHECK();
                }
                // ---- segments longer than a CTA sort: split into ordered
                //      id ranges that each fit one (k_big_split), sorted as
                //      sub-segments; those that do not split go to one
                //      device-wide keys-only radix sort
                unsigned int n_big = 0;
                if (nbm[0]) {
                    const unsigned int nlong = nbm[0];
                    DevBuf<unsigned long long> rk2(h.total, s), d_off((size_t)nlong * SPLIT_MAXB, s);
                    DevBuf<uint32_t> d_cnt((size_t)nlong * SPLIT_MAXB, s),
                        d_q((size_t)nlong * SPLIT_MAXB, s);
                    k_big_split<<<nlong, 256, 0, s>>>(lists.p + 3 * nslots, counts_p, offsets_p,
                                                     rkeys.p, rk2.p, bigc.p, d_off.p, d_cnt.p,
                                                     d_q.p, ctr_p);
                    DTS_LAUNCH_CHECK();
                    unsigned int nd[3] = {0, 0, 0};            // n_desc, n_dskew, n_bigfb
                    DTS_CUDA(cudaMemcpyAsync(nd, &ctr_p->n_desc, sizeof(nd),
                                             cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                    const SegDesc ds{d_off.p, d_cnt.p, d_q.p};
                    if (nd[0]) {
                        DevBuf<uint32_t> dskew(nd[0], s);
                        k_seg_bucket<1024, 16, 1, true><<<nd[0], 1024, SEG_CAP * 12, s>>>(
                            nullptr, counts_p, offsets_p, rk2.p, src, qmap, qid_base, fin, dskew.p,
                            ctr_p, ds);
                        DTS_LAUNCH_CHECK();
                        unsigned int nsk = 0;
                        DTS_CUDA(cudaMemcpyAsync(&nsk, &ctr_p->n_dskew, sizeof(nsk),
                                                 cudaMemcpyDeviceToHost, s));
                        DTS_CUDA(cudaStreamSynchronize(s));
                        if (nsk) {
                            k_seg_radix<1024, 16, 1, true><<<nsk, 1024, SEG_CAP * 8, s>>>(
                                dskew.p, counts_p, offsets_p, rk2.p, src, qmap, qid_base, eb, fin,
                                ds);
                            DTS_LAUNCH_CHECK();
                        }
                        DTS_CUDA(cudaStreamSynchronize(s));    // before the scratch goes
                    }
                    n_big = nd[2];
                }
                if (n_big) {
                    // ---- segments longer than a CTA sort: one device-wide
                    //      keys-only radix sort over those only
                    DevBuf<unsigned long long> bigoff(nq + 1, s);
                    scan_exclusive_u32_to_u64(bigc.p, bigoff.p, nq, s);
                    unsigned long long nb = 0;
                    DTS_CUDA(cudaMemcpyAsync(&nb, bigoff.p + nq, sizeof(nb),
                                             cudaMemcpyDeviceToHost, s));
                    DTS_CUDA(cudaStreamSynchronize(s));
                    // key bits: query, entry id (caller ids: 32 bits), slot
                    const int qb = bits_for(nq - 1), eb = idx->eid_bits;
                    const int sb = std::max(1, bits_for((unsigned long long)h.c.max_count - 1));
                    if (qb + eb + sb > 64)
                        throw Error(DTS_ENOTSUP, "long result segments: sort key exceeds 64 bits");
                    DevBuf<unsigned long long> k1(nb, s), k2(nb, s);
                    k_big_keys<<<blocks((size_t)nq * 32, 256), 256, 0, s>>>(
                        (uint32_t)nq, bigc.p, bigoff.p, offsets_p, rkeys.p, eb, sb, k1.p);
                    DTS_LAUNCH_CHECK();
                    const unsigned long long* sk =
                        radix_sort_keys(k1.p, k2.p, nb, sb, sb + eb + qb, s);
                    k_big_place<<<blocks(nb, 256), 256, 0, s>>>(sk, nb, eb, sb, bigoff.p,
                                                               offsets_p, rkeys.p, src, qmap, qid_base,
                                                               fin);
                    DTS_LAUNCH_CHECK();
                }
            }
            tm.mark();
            DTS_CUDA(cudaStreamSynchronize(s));
        } catch (...) {
            cudaStreamSynchronize(s);
            cache_free(fin);
            throw;
        }
        out->results = fin;
        out->count = (size_t)h.total;
    } else {
        tm.mark();
        tm.mark();
    }
    tr.mark("done");
    if (local.time_kernels >= 2) {
        local.timer_slot = tm.handle;
    } else if (local.time_kernels) {
        DTS_CUDA(cudaStreamSynchronize(s));
        local.ms_prep = tm.ms(0);
        local.ms_count = tm.ms(1);
        local.ms_scan = tm.ms(2);
        local.ms_scatter = tm.ms(3);
        local.ms_canon = tm.ms(4);
    }
    if (stats) *stats = local;
}

void search_read_times(dts_search_stats* st) {
    int dev = 0;
    DTS_CUDA(cudaGetDevice(&dev));
    TimerRing& r = timer_ring(dev);
    const uint32_t h = st->timer_slot, i = h % TIMER_SETS;
    if (h >= r.next || r.next - h > TIMER_SETS || !r.made[i])
        throw Error(DTS_EINVAL, "timer slot recycled or not from this thread and device");
    const uint32_t rec = r.rec[i];
    if (rec) DTS_CUDA(cudaEventSynchronize(r.ev[i][31 - __builtin_clz(rec)]));
    float* out[5] = {&st->ms_prep, &st->ms_count, &st->ms_scan, &st->ms_scatter, &st->ms_canon};
    for (int j = 0; j < 5; ++j) {
        float t = 0.f;
        if (((rec >> j) & 3u) == 3u) DTS_CUDA(cudaEventElapsedTime(&t, r.ev[i][j], r.ev[i][j + 1]));
        *out[j] = t;
    }
}

void query_costs_device(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                        uint32_t block, unsigned long long* out, cudaStream_t s, uint32_t stride) {
    if (block == 0) throw Error(DTS_EINVAL, "block must be >= 1");
    if (stride == 0) throw Error(DTS_EINVAL, "stride must be >= 1");
    if (idx->ooc) throw Error(DTS_ENOTSUP, "query costs of an index over temporal shards");
    const size_t nb = (nq + block - 1) / block;
    if (nb) DTS_CUDA(cudaMemsetAsync(out, 0, nb * sizeof(unsigned long long), s));
    if (nq == 0 || idx->n == 0) return;
    if (idx->ready) DTS_CUDA(cudaStreamWaitEvent(s, idx->ready, 0));
    k_query_costs<<<blocks((nq + stride - 1) / stride, PT), PT, 0, s>>>(
        reinterpret_cast<const double4*>(Q_dev), (uint32_t)nq, d, idx->gp, idx->ht,
        idx->bin_t0min, idx->bin_t1max, idx->bin_start, idx->method, idx->sb, block, stride, out);
    DTS_LAUNCH_CHECK();
}

namespace {
__global__ void __launch_bounds__(PT) k_result_keys(const dts_result* __restrict__ r,
                                                   unsigned long long n,
                                                   unsigned long long* __restrict__ keys,
                                                   uint32_t* __restrict__ vals) {
    const unsigned long long k = (unsigned long long)blockIdx.x * PT + threadIdx.x;
    if (k >= n) return;
    keys[k] = ((unsigned long long)r[k].query_id << 32) | r[k].entry_id;
    vals[k] = (uint32_t)k;
}
__global__ void __launch_bounds__(PT) k_result_gather(const dts_result* __restrict__ r,
                                                     const uint32_t* __restrict__ vals,
                                                     unsigned long long n,
                                                     dts_result* __restrict__ out) {
    const unsigned long long k = (unsigned long long)blockIdx.x * PT + threadIdx.x;
    if (k < n) out[k] = r[vals[k]];
}
}  // namespace

// Canonical (query_id, entry_id) order of an arbitrary result array, e.g.
// the concatenated outputs of temporal shards of D: one
// stable radix sort of the 64-bit (query, entry) keys, then a gather.
void canonicalize_device(dts_result* r, size_t n, cudaStream_t s) {
    if (n <= 1) return;
    if (n >= (size_t(1) << 32)) throw Error(DTS_ENOTSUP, "more than 2^32 results to sort");
    DevBuf<unsigned long long> k1(n, s), k2(n, s);
    DevBuf<uint32_t> v1(n, s), v2(n, s);
    DevBuf<dts_result> tmp(n, s);
    k_result_keys<<<blocks(n, PT), PT, 0, s>>>(r, n, k1.p, v1.p);
    DTS_LAUNCH_CHECK();
    radix_sort_pairs(k1.p, v1.p, k2.p, v2.p, n, 64, s);
    k_result_gather<<<blocks(n, PT), PT, 0, s>>>(r, v1.p, n, tmp.p);
    DTS_LAUNCH_CHECK();
    DTS_CUDA(cudaMemcpyAsync(r, tmp.p, n * sizeof(dts_result), cudaMemcpyDeviceToDevice, s));
    DTS_CUDA(cudaStreamSynchronize(s));
}

}  // namespace dts
