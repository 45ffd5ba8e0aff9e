// internal.cuh -- shared internals of libdts (CUDA side only; never included
// by the oracle).  Layouts, grid parameters, error plumbing and the device
// helpers used by both the index builder and the search kernels.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/dts.h"

namespace dts {

// ------------------------------------------------------------ host trace
// Host timeline of one call (DTS_TRACE=1: one line on stderr per call, the
// microseconds from the call's entry to each mark); a diagnostic of the
// per-call host cost, off by default.
struct HostTrace {
    static bool enabled() {
        static const bool on = [] {
            const char* e = std::getenv("DTS_TRACE");
            return e && e[0] == '1';
        }();
        return on;
    }
    const char* tag;
    bool on = enabled();
    int k = 0;
    const char* what[16];
    std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now(), t[16];
    explicit HostTrace(const char* name) : tag(name) {}
    void mark(const char* w) {
        if (on && k < 16) { what[k] = w; t[k++] = std::chrono::steady_clock::now(); }
    }
    ~HostTrace() {
        if (!on) return;
        std::fprintf(stderr, "[dts trace] %s", tag);
        for (int i = 0; i < k; ++i)
            std::fprintf(stderr, " %s=%.1f", what[i],
                         std::chrono::duration<double, std::micro>(t[i] - t0).count());
        std::fprintf(stderr, "\n");
    }
};

// ---------------------------------------------------------------- errors
struct Error : std::runtime_error {
    dts_status status;
    Error(dts_status s, const std::string& m) : std::runtime_error(m), status(s) {}
};

void set_last_error(const std::string& msg);

#define DTS_CUDA(call)                                                              \
    do {                                                                            \
        cudaError_t _e = (call);                                                    \
        if (_e != cudaSuccess) {                                                    \
            if (_e == cudaErrorMemoryAllocation)                                    \
                throw ::dts::Error(DTS_ENOMEM, std::string(#call) + ": " +          \
                                   cudaGetErrorString(_e));                         \
            throw ::dts::Error(DTS_ECUDA, std::string(#call) + ": " +               \
                               cudaGetErrorString(_e));                             \
        }                                                                           \
    } while (0)

// Every kernel launch is followed by DTS_LAUNCH_CHECK(), which also counts it
// (dts_kernel_launches(), used by the benchmark's gpu_launches claim).
extern std::atomic<unsigned long long> g_launches;
#define DTS_LAUNCH_CHECK()                                                          \
    do {                                                                            \
        ::dts::g_launches.fetch_add(1, std::memory_order_relaxed);                  \
        DTS_CUDA(cudaGetLastError());                                               \
    } while (0)

// Device-side invariant checks, compiled in only for the checked build
// (DTS_NVCC_EXTRA=-DDTS_CHECKED, scripts/gpu_checked.sh): a failed check
// prints its condition and traps, which fails the calling test.
#ifdef DTS_CHECKED
#define DTS_DCHECK(c)                                                               \
    do {                                                                            \
        if (!(c)) {                                                                 \
            printf("DTS_DCHECK failed %s:%d: %s\n", __FILE__, __LINE__, #c);       \
            __trap();                                                               \
        }                                                                           \
    } while (0)
#else
#define DTS_DCHECK(c) do {} while (0)
#endif

// Stream-ordered device buffer (pool allocator; freed on scope exit).
template <typename T>
struct DevBuf {
    T* p = nullptr;
    size_t n = 0;
    cudaStream_t s = nullptr;
    DevBuf() = default;
    DevBuf(size_t count, cudaStream_t st) { alloc(count, st); }
    void alloc(size_t count, cudaStream_t st) {
        release();
        s = st;
        n = count;
        if (count) DTS_CUDA(cudaMallocAsync((void**)&p, count * sizeof(T), st));
    }
    void release() {
        if (p) cudaFreeAsync(p, s);
        p = nullptr;
        n = 0;
    }
    T* detach() { T* r = p; p = nullptr; n = 0; return r; }
    ~DevBuf() { release(); }
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
};

// ---------------------------------------------------------------- layout
// Entry segments in the index live in key order as one 64-byte record each,
//   (t_start, t_end, x_start, vx, y_start, vy, z_start, vz),
// read and written as two 256-bit accesses, with v = (end - start) /
// (t_end - t_start) precomputed at build (0 for a zero-duration segment,
// which can never overlap strictly in time).  The position at time t is
// start + (t - t_start) * v.  (Four 16-byte double2 streams instead were
// measured slower on C4 in round 1: gather 0.765 vs 0.759 ms, pass 1 0.802
// vs 0.742.)
struct SegSoA {
    double2* rec;    // 4 double2 per sorted position
    uint32_t* eid;   // caller's entry id of each sorted position
#ifdef __CUDACC__
    __device__ __forceinline__ const double2* at(size_t p) const { return rec + 4 * p; }
    // the record of sorted position p (two 256-bit loads)
    __device__ __forceinline__ void load4(size_t p, double2& st, double2& sx, double2& sy,
                                          double2& sz) const;
    __device__ __forceinline__ void store4(size_t p, double2 st, double2 sx, double2 sy,
                                           double2 sz) const;
#endif
};

static constexpr unsigned long long EMPTY_KEY = ~0ull;

// Hash slot of one non-empty BLOCK of 8 consecutive keys (key >> 3): 8
// x-adjacent cells of a row (a block may straddle two rows).  The block's
// entries are the sorted positions [start, start + cum[7]); those of key
// offset j are [start + cum[j-1], start + cum[j]) (cum[-1] = 0).  When the
// block holds more than 65535 entries, big = 1, cum is unused and the block
// is one run [start, end) with end = start + cum32 (exact superset: the
// refinement filters).  32 bytes, one 256-bit load; two per 64-byte bucket.
struct __align__(32) BlockSlot {
    unsigned long long key;
    uint32_t start;
    uint32_t big;
    uint16_t cum[8];
};

// Grid parameters (passed by value to kernels).
struct GridParams {
    double tmin;        // temporal origin  (t_min of P:L76)
    double inv_b;       // 1 / bin width
    double b;           // bin width        (b of P:L76)
    double maxdur;      // max(t_end - t_start) over D
    double o[3];        // spatial origin (per-axis min over D)
    double w[3];        // cell width per axis
    double inv_w[3];
    double half_ext[3]; // half of the max per-axis extent
    int32_t m;          // bins
    int32_t nc[3];      // cells per axis
    unsigned long long cells_per_bin;  // nc0*nc1*nc2
};

struct HashTable {
    void* slots;               // BlockSlot, 2 per 64-byte bucket
    unsigned long long nbuckets;   // buckets (any count: not a power of two)
    __host__ __device__ BlockSlot* blocks() const { return static_cast<BlockSlot*>(slots); }
    __host__ __device__ unsigned long long nslots() const { return 2ull * nbuckets; }
};

// GPUSpatioTemporal subbins (P:L86-P:L92): per dimension a, v[a] subbins of
// width >= the largest entry extent in a; ids[a] holds the sorted positions of
// the entries overlapping subbin j of bin i, chunks in (j, i) lexicographic
// order; chunk (j, i) is ids[a][dir[a][j*m + i] .. dir[a][j*m + i + 1]).
struct SubbinIndex {
    double o[3];
    double inv_w[3];
    int32_t v[3];
    int32_t m;
    const uint32_t* ids[3];
    const uint32_t* dir[3];
    // the entry records of ids[a], in the same order (64 bytes per slot, two
    // 256-bit loads): a subbin chunk streams its candidates contiguously
    // instead of one dependent random record read per id
    const double4* rec[3];
};

__device__ __forceinline__ int32_t subbin_of(const SubbinIndex& s, int a, double x) {
    double f = floor((x - s.o[a]) * s.inv_w[a]);
    if (!(f > 0.0)) return 0;
    if (f >= (double)(s.v[a] - 1)) return s.v[a] - 1;
    return (int32_t)f;
}

// ---------------------------------------------------------------- device helpers
// Bucketed open addressing, 64-byte buckets.  Keys are row-major with x
// fastest, so x-adjacent cells share a block: blocks of 8 keys (k >> 3, one
// 32-byte slot per block) are hashed into buckets of two slots.  A stencil
// row of three cells then reads one or two buckets.  (One 16-byte slot per
// cell, four per bucket, measured slower in round 1: insert 0.56 vs 0.44 ms,
// pass 1 0.80 vs 0.65 ms on C4.)  An item sits in the
// first bucket, from its home on, that had a free slot when it was inserted
// (no deletions), so a lookup stops at the first bucket holding it or a
// free slot -- almost always the home bucket.
// Home bucket: a Fibonacci hash of the block key mapped onto [0, nbuckets)
// by a multiply-shift range reduction (the table is sized to the load
// factor exactly, not rounded up to a power of two: with power-of-two sizes
// the same load target gave anywhere from 3.3 to 6.6 slots per block).
__device__ __forceinline__ unsigned long long bucket_of(unsigned long long group,
                                                        const HashTable& ht) {
    const unsigned long long h = (group * 0x9E3779B97F4A7C15ull) >> 32;   // 32 mixed bits
    return (h * ht.nbuckets) >> 32;
}
__device__ __forceinline__ unsigned long long next_bucket(unsigned long long b,
                                                          const HashTable& ht) {
    return b + 1 == ht.nbuckets ? 0ull : b + 1;
}

__device__ __forceinline__ int32_t bin_of(const GridParams& g, double t) {
    double f = floor((t - g.tmin) * g.inv_b);
    if (!(f > 0.0)) return 0;                       // also maps NaN to 0
    if (f >= (double)(g.m - 1)) return g.m - 1;
    return (int32_t)f;
}

__device__ __forceinline__ int32_t cell_of(const GridParams& g, int a, double v) {
    double f = floor((v - g.o[a]) * g.inv_w[a]);
    if (!(f > 0.0)) return 0;
    if (f >= (double)(g.nc[a] - 1)) return g.nc[a] - 1;
    return (int32_t)f;
}

__device__ __forceinline__ unsigned long long make_key(const GridParams& g, int32_t bin,
                                                       int32_t cx, int32_t cy, int32_t cz) {
    return (unsigned long long)bin * g.cells_per_bin +
           ((unsigned long long)cz * (unsigned long long)g.nc[1] + (unsigned long long)cy) *
               (unsigned long long)g.nc[0] +
           (unsigned long long)cx;
}

// ---------------------------------------------------------------- outliers
// Entries far longer in space or time than the rest ("outliers": extent or
// duration above 8x the sample mean) are not filed by MBB midpoint -- their
// extent would widen every query's stencil and their duration every
// query's bin range.  Each is filed instead as copies along its path: for
// every bin j its time overlaps, the time inside the bin is cut into S
// sub-slices of about one cell of travel, and the copy keys are the cells of
// each sub-slice's box.  A query meets the copies in its stencil; the search
// keeps a hit on a copy only from the canonical copy: the least key among the
// sub-slice boxes of the first probed bin whose boxes meet the query's
// stencil (outlier_canonical in search.cu).  Build and search derive the
// boxes with this one function from the same record values, so they agree
// bit for bit.
struct ORec {
    double t0, t1;
    double x[3], v[3];   // velocity form: position at t = x + (t - t0) v
};

template <typename F>
__device__ __forceinline__ void outlier_boxes(const GridParams& g, const ORec& o, int32_t j,
                                              int32_t jo0, int32_t jo1, F&& f) {
    const double eps = 1e-12 * (fabs(g.tmin) + fabs(o.t0) + fabs(o.t1) + g.b);
    const double ts = (j == jo0) ? o.t0 : fmax(o.t0, g.tmin + (double)j * g.b - eps);
    const double te = (j == jo1) ? o.t1 : fmin(o.t1, g.tmin + (double)(j + 1) * g.b + eps);
    double cross = 0.0;
#pragma unroll
    for (int a = 0; a < 3; ++a) cross = fmax(cross, fabs(o.v[a]) * (te - ts) * g.inv_w[a]);
    const int S = (int)fmin(64.0, fmax(1.0, ceil(cross)));
    for (int k = 0; k < S; ++k) {
        const double ta = ts + (te - ts) * (double)k / (double)S;
        const double tb = (k + 1 == S) ? te : ts + (te - ts) * (double)(k + 1) / (double)S;
        int32_t lo[3], hi[3];
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            const double pa = o.x[a] + (ta - o.t0) * o.v[a];
            const double pb = o.x[a] + (tb - o.t0) * o.v[a];
            const double sl = 1e-12 * (fabs(pa) + fabs(pb) + g.w[a]);
            lo[a] = cell_of(g, a, fmin(pa, pb) - sl);
            hi[a] = cell_of(g, a, fmax(pa, pb) + sl);
        }
        f(lo, hi);
    }
}

// Outlier state of an index (device pointers; okeys == NULL: no outliers).
struct OutlierIndex {
    const unsigned long long* okeys;   // sorted packed keys (key << shift | row) per position
    const uint32_t* obits;             // bitmap over sorted positions: 1 = an outlier's copy
    int shift;
};

// 256-bit read-only load (sm_100: LDG.E.256; one 32-byte sector per lane).
__device__ __forceinline__ double4 ld256(const double4* p) {
    double4 v;
    asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
                 : "=d"(v.x), "=d"(v.y), "=d"(v.z), "=d"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ ulonglong4 ld256u(const void* p) {
    ulonglong4 v;
    asm("ld.global.nc.v4.u64 {%0,%1,%2,%3}, [%4];"
                 : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p));
    return v;
}

// Both 256-bit halves of a record, issued together: `volatile` keeps the
// compiler from sinking the second load behind the refinement's temporal
// test (it did: one more dependent memory round trip per candidate).
__device__ __forceinline__ void ld512v(const double4* p, double4& a, double4& b) {
    asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%8];\n\t"
                 "ld.global.nc.v4.f64 {%4,%5,%6,%7}, [%8+32];"
                 : "=d"(a.x), "=d"(a.y), "=d"(a.z), "=d"(a.w), "=d"(b.x), "=d"(b.y), "=d"(b.z),
                   "=d"(b.w)
                 : "l"(p));
}

__device__ __forceinline__ void SegSoA::load4(size_t p, double2& st, double2& sx, double2& sy,
                                              double2& sz) const {
    const double4* r = reinterpret_cast<const double4*>(rec + 4 * p);
    double4 a, b;
    ld512v(r, a, b);
    st = make_double2(a.x, a.y);
    sx = make_double2(a.z, a.w);
    sy = make_double2(b.x, b.y);
    sz = make_double2(b.z, b.w);
}
__device__ __forceinline__ void SegSoA::store4(size_t p, double2 st, double2 sx, double2 sy,
                                               double2 sz) const {
    double* r = reinterpret_cast<double*>(rec + 4 * p);
    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(r), "d"(st.x), "d"(st.y),
                 "d"(sx.x), "d"(sx.y) : "memory");
    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(r + 4), "d"(sy.x), "d"(sy.y),
                 "d"(sz.x), "d"(sz.y) : "memory");
}

// Monotone map of doubles to unsigned 64-bit integers (for atomic min/max).
__device__ __forceinline__ unsigned long long ordered_bits(double x) {
    unsigned long long u = (unsigned long long)__double_as_longlong(x);
    return (u & 0x8000000000000000ull) ? ~u : (u | 0x8000000000000000ull);
}
__host__ __device__ inline double from_ordered_bits(unsigned long long u) {
    unsigned long long v = (u & 0x8000000000000000ull) ? (u & ~0x8000000000000000ull) : ~u;
#ifdef __CUDA_ARCH__
    return __longlong_as_double((long long)v);
#else
    double d;
    memcpy(&d, &v, 8);
    return d;
#endif
}

// ---------------------------------------------------------------- primitives (prims.cu)
// Exclusive scan of n values; out has n + 1 entries, out[n] = total.
void scan_exclusive_u32_to_u32(const uint32_t* in, uint32_t* out, size_t n, cudaStream_t s);
void scan_exclusive_u32_to_u64(const uint32_t* in, unsigned long long* out, size_t n,
                               cudaStream_t s, unsigned long long* total_out = nullptr);

// Stable LSD radix sort of (key, value) pairs on key bits [0, nbits).
// Sorts in place from the caller's view: on return keys/vals hold the result.
// keys_tmp / vals_tmp are caller-provided scratch of n entries each.
void radix_sort_pairs(unsigned long long* keys, uint32_t* vals, unsigned long long* keys_tmp,
                      uint32_t* vals_tmp, size_t n, int nbits, cudaStream_t s);

// Stable LSD radix sort of u64 keys on bits [lo, hi) only (keys-only: a
// payload packed in the bits below lo rides along untouched; since the input
// is in payload order, sorting on [lo, hi) equals a stable sort by the key).
// Returns the buffer (keys or tmp) that holds the sorted keys.
unsigned long long* radix_sort_keys(unsigned long long* keys, unsigned long long* tmp, size_t n,
                                    int lo, int hi, cudaStream_t s);

int bits_for(unsigned long long max_value);

// Digit layout of a multi-pass onesweep sort: pass p sorts the digit of width
// bits[p] (8 or 9) at bit shift[p]; its histogram is hist[p * 512 + digit].
constexpr int OS_MAXPASS = 8;
constexpr int OS_HSTRIDE = 512;
struct PassPlan {
    int npass;
    int shift[OS_MAXPASS];
    int bits[OS_MAXPASS];
};
// As few passes as 9-bit digits allow for bits [lo, hi) (8-bit where enough).
PassPlan plan_passes(int lo, int hi, bool allow9);
// Whether n keys go through the onesweep sort (else hist + scan + scatter).
bool radix_onesweep(size_t n);
// Keys-only onesweep sort by the plan, with the per-pass digit counts
// already accumulated in hist (npass x 512, e.g. by the kernel that wrote the
// keys).  Returns the buffer (keys or tmp) holding the sorted keys; with
// rows_out the last pass writes only (key & row_mask) of each sorted key
// there (a packed (key, row) sort that only needs the order) and returns NULL.
unsigned long long* radix_sort_keys_hist(unsigned long long* keys, unsigned long long* tmp,
                                         size_t n, const PassPlan& plan, uint32_t* hist,
                                         cudaStream_t s, uint32_t* rows_out = nullptr,
                                         unsigned long long row_mask = 0);

// Device block cache (alloc.cu) for memory that outlives one API call.
void* cache_alloc(size_t bytes);
void cache_free(void* p);
int cache_device(void* p);          // owning device of a live block, -1 if not ours

// Saves the caller's current device and restores it on scope exit (every
// entry point of the C ABI runs under one: the library switches to the
// index's device, the caller's thread state is left as it was).
struct DeviceGuard {
    int prev = -1;
    DeviceGuard() { if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); prev = -1; } }
    ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
    DeviceGuard(const DeviceGuard&) = delete;
    DeviceGuard& operator=(const DeviceGuard&) = delete;
};

}  // namespace dts

namespace dts {
// Temporal shards of an entry database larger than the device budget (ooc.cu).
struct OocShard {
    size_t n = 0;
    double t0min = 0, t1max = 0;   // min t_start, max t_end of the shard's entries
};
struct OocIndex {
    dts_segment* D_h = nullptr;    // pinned, shards contiguous
    uint32_t* ids_h = nullptr;     // pinned, reported entry id per row
    uint32_t* traj_h = nullptr;    // pinned, trajectory id per row (optional)
    std::vector<OocShard> shards;
    std::vector<size_t> off;       // first row of each shard
    dts_index_params p{};          // parameters of the per-shard builds
};
}  // namespace dts

// The opaque index (definition shared by build.cu, search.cu and api.cu).
struct dts_index {
    int device = 0;
    uint64_t n = 0;
    dts::GridParams gp{};
    dts::SegSoA soa{};
    dts::HashTable ht{};
    unsigned long long n_cells = 0;
    double* bin_t0min = nullptr;   // per bin: min t_start (bin extent)
    double* bin_t1max = nullptr;   // per bin: max t_end   (B_end of P:L76)
    uint32_t* bin_start = nullptr; // m + 1 sorted-position offsets of the bins
    void* block = nullptr;         // single device allocation backing the arrays above
    double max_ext[3] = {0, 0, 0};
    float ms_build = 0.f;
    float ms_phase[5] = {0, 0, 0, 0, 0};   // bounds, keys, sort, gather, insert
    bool fused_keys = false;       // sampled grid + one-read bounds/keys/histograms
    unsigned long long hash_items = 0;
    cudaEvent_t ev[7] = {};        // build phase events (index_times)
    int nev = 0;
    bool timed = false;
    cudaEvent_t ready = nullptr;   // end of the build (= ev[nev - 1])
    int key_bits = 0;
    uint32_t method = 0;           // dts_method
    dts::SubbinIndex sb{};         // DTS_METHOD_SUBBIN only
    uint32_t* sb_block[3] = {nullptr, nullptr, nullptr};   // ids + dir per dimension
    double4* sb_rec[3] = {nullptr, nullptr, nullptr};      // records of ids, per dimension
    uint64_t sb_len[3] = {0, 0, 0};
    uint32_t* etraj = nullptr;     // trajectory id per sorted position (optional)
    // spill-buffer size hint (records): the largest output a search of this
    // index has produced after its spill buffer filled (search.cu)
    mutable std::atomic<unsigned long long> spill_hint{0};
    // results per query of the last search of this index: the next search's
    // speculative pass 2 gets that rate x its queries plus an eighth (0: none
    // yet)
    mutable std::atomic<double> result_hint{0.0};
    int eid_bits = 32;             // bits of the largest reported entry id
    dts::OutlierIndex out{};       // long-segment copies (build.cu), okeys NULL if none
    void* out_block = nullptr;     // backing memory of out (cache)
    unsigned long long n_outliers = 0, n_copies = 0;
    dts::OocIndex* ooc = nullptr;  // set: D lives in pinned host temporal shards
};

namespace dts {
void build_index_device(dts_index* idx, const dts_segment* D_dev, size_t n,
                        const dts_index_params& p, cudaStream_t s);
// Waits for the end of the build and fills ms_build / ms_phase.
void index_times(dts_index* idx);
struct SearchOut {
    dts_result* results = nullptr;   // device, cudaMalloc'd (caller owns)
    size_t count = 0;
};
// Thrown by search_device when the results would not fit in device memory
// (or exceed max_results): carries the per-query counts (query-id order) so a
// host caller can stream the search in query chunks.
struct ResultsTooLarge : Error {
    unsigned long long total;
    std::vector<uint32_t> counts;
    explicit ResultsTooLarge(unsigned long long t)
        : Error(DTS_ENOMEM, "results (" + std::to_string(t) +
                                ") do not fit in device memory; dts_search (host) streams them "
                                "in query chunks"),
          total(t) {}
};
void search_device(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                   uint32_t qid_base, cudaStream_t s, SearchOut* out, dts_search_stats* stats,
                   unsigned long long max_results = ~0ull, const uint32_t* qmap = nullptr,
                   const uint32_t* qtraj = nullptr, bool exclude_same_traj = false,
                   bool count_only = false, uint32_t* counts_out = nullptr);
// Per-query candidate counts summed per block of `block` queries (search.cu).
void search_read_times(dts_search_stats* stats);
void query_costs_device(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                        uint32_t block, unsigned long long* out, cudaStream_t s,
                        uint32_t stride = 1);
// Trajectory-level merge (traj.cu); output in cache_alloc'd device memory.
void merge_trajectories_device(const dts_result* r, size_t n, const uint32_t* qtraj,
                               size_t nqid, const uint32_t* etraj, size_t neid,
                               cudaStream_t s, dts_traj_result** out, size_t* count);
// Sort results in device memory by (query_id, entry_id), in place.
void canonicalize_device(dts_result* r, size_t n, cudaStream_t s);
// Device memory of an index (after its build has finished) back to the cache.
void free_index_arrays(dts_index* idx);
// Entry databases larger than the budget (ooc.cu).
uint64_t index_bytes_estimate(size_t n);
void ooc_build(dts_index* idx, const dts_segment* D_host, size_t n, const dts_index_params& p,
               cudaStream_t s);
void ooc_free(OocIndex* o);
void ooc_search(const dts_index* idx, const dts_segment* Q_dev, size_t nq, double d,
                uint32_t qid_base, cudaStream_t s, SearchOut* out, dts_search_stats* stats,
                const uint32_t* qmap, const uint32_t* qtraj, bool excl, bool count_only,
                uint32_t* counts_out);
}  // namespace dts
