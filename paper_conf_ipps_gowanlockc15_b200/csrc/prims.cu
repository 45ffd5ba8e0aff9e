// prims.cu -- device-wide primitives written for this library: exclusive
// scan (reduce / scan-of-partials / downsweep) and a stable LSD radix sort of
// (u64 key, u32 value) pairs with warp-level match-based ranking.
//
// These implement the "radix sort and prefix scan" of the index builder
// (BASELINE.json north_star) and the exclusive scan of
// per-query result counts of the two-pass compaction (§8(a6)).
#include <algorithm>
#include <cstdlib>

#include "internal.cuh"

namespace dts {

int bits_for(unsigned long long v) {
    int b = 0;
    while (v) { ++b; v >>= 1; }
    return b;
}

// ============================================================== scan
namespace {
constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 4;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;   // 1024

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T u = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += u;
    }
    return v;
}

// Block-wide exclusive scan of one value per thread; returns the exclusive
// prefix and writes the block total to *total.
template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* total) {
    __shared__ T warp_sums[SCAN_THREADS / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T inc = warp_inclusive_scan(v);
    if (lane == 31) warp_sums[warp] = inc;
    __syncthreads();
    if (warp == 0) {
        T s = (lane < SCAN_THREADS / 32) ? warp_sums[lane] : T(0);
        s = warp_inclusive_scan(s);
        if (lane < SCAN_THREADS / 32) warp_sums[lane] = s;
    }
    __syncthreads();
    T warp_prefix = warp ? warp_sums[warp - 1] : T(0);
    *total = warp_sums[SCAN_THREADS / 32 - 1];
    __syncthreads();
    return warp_prefix + inc - v;
}

template <typename Tin, typename Tout>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_reduce(const Tin* __restrict__ in, size_t n,
                                                              Tout* __restrict__ sums) {
    size_t base = (size_t)blockIdx.x * SCAN_TILE;
    Tout s = 0;
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; ++i) {
        size_t idx = base + (size_t)i * SCAN_THREADS + threadIdx.x;
        if (idx < n) s += (Tout)in[idx];
    }
    Tout total;
    block_exclusive_scan<Tout>(s, &total);
    if (threadIdx.x == 0) sums[blockIdx.x] = total;
}

// Downsweep: out[i] = prefix(block) + exclusive scan inside the block.
// prefix == nullptr means a single-block scan; then out[n] = total.
template <typename Tin, typename Tout>
__global__ void __launch_bounds__(SCAN_THREADS) k_scan_down(const Tin* __restrict__ in, size_t n,
                                                            const Tout* __restrict__ prefix,
                                                            Tout* __restrict__ out,
                                                            Tout* __restrict__ total_out) {
    size_t base = (size_t)blockIdx.x * SCAN_TILE + (size_t)threadIdx.x * SCAN_ITEMS;
    Tout v[SCAN_ITEMS];
    Tout s = 0;
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; ++i) {
        size_t idx = base + i;
        v[i] = idx < n ? (Tout)in[idx] : Tout(0);
        s += v[i];
    }
    Tout total;
    Tout run = block_exclusive_scan<Tout>(s, &total);
    Tout bp = prefix ? prefix[blockIdx.x] : Tout(0);
    run += bp;
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; ++i) {
        size_t idx = base + i;
        if (idx < n) out[idx] = run;
        run += v[i];
    }
    if (prefix == nullptr && threadIdx.x == 0) {
        out[n] = total;
        if (total_out) *total_out = total;
    }
    if (prefix != nullptr && blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
        out[n] = prefix[gridDim.x];
        if (total_out) *total_out = prefix[gridDim.x];
    }
}

template <typename Tin, typename Tout>
void scan_exclusive(const Tin* in, Tout* out, size_t n, cudaStream_t s, Tout* total_out = nullptr) {
    if (n <= (size_t)SCAN_TILE) {
        k_scan_down<Tin, Tout><<<1, SCAN_THREADS, 0, s>>>(in, n, nullptr, out, total_out);
        DTS_LAUNCH_CHECK();
        return;
    }
    size_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    DevBuf<Tout> sp(2 * nb + 1, s);                  // block sums, then their scan
    Tout* const sums = sp.p;
    Tout* const pre = sp.p + nb;
    k_scan_reduce<Tin, Tout><<<(unsigned)nb, SCAN_THREADS, 0, s>>>(in, n, sums);
    DTS_LAUNCH_CHECK();
    scan_exclusive<Tout, Tout>(sums, pre, nb, s);
    k_scan_down<Tin, Tout><<<(unsigned)nb, SCAN_THREADS, 0, s>>>(in, n, pre, out, total_out);
    DTS_LAUNCH_CHECK();
}
}  // namespace

void scan_exclusive_u32_to_u32(const uint32_t* in, uint32_t* out, size_t n, cudaStream_t s) {
    scan_exclusive<uint32_t, uint32_t>(in, out, n, s);
}
void scan_exclusive_u32_to_u64(const uint32_t* in, unsigned long long* out, size_t n,
                               cudaStream_t s, unsigned long long* total_out) {
    scan_exclusive<uint32_t, unsigned long long>(in, out, n, s, total_out);
}
// ============================================================== radix sort
namespace {
constexpr int RS_THREADS = 256;
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_ITEMS = 8;                       // per thread
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;    // 2048 keys per CTA

// Per-tile digit histogram; counts laid out digit-major so that one
// exclusive scan yields every (digit, tile) output offset.
template <int BITS>
__global__ void __launch_bounds__(RS_THREADS) k_rs_hist(const unsigned long long* __restrict__ keys,
                                                        size_t n, int shift,
                                                        uint32_t* __restrict__ counts,
                                                        uint32_t ntiles) {
    constexpr int RADIX = 1 << BITS;
    __shared__ uint32_t h[RADIX];
    for (int j = threadIdx.x; j < RADIX; j += RS_THREADS) h[j] = 0;
    __syncthreads();
    size_t base = (size_t)blockIdx.x * RS_TILE;
#pragma unroll
    for (int i = 0; i < RS_ITEMS; ++i) {
        size_t idx = base + (size_t)i * RS_THREADS + threadIdx.x;
        if (idx < n) atomicAdd(&h[(uint32_t)(keys[idx] >> shift) & (RADIX - 1)], 1u);
    }
    __syncthreads();
    for (int j = threadIdx.x; j < RADIX; j += RS_THREADS)
        counts[(size_t)j * ntiles + blockIdx.x] = h[j];
}

// Stable scatter.  Warp w of a tile owns the contiguous chunk
// [tile + w*256, tile + (w+1)*256); within a warp items are visited in
// (item, lane) order = input order, ranked with __match_any_sync and
// warp-private digit counters; a cross-warp prefix per digit then orders the
// chunks.  The tile is staged in digit order in shared memory and written
// out with consecutive threads on consecutive output positions.
template <int BITS, bool VALS>
__global__ void __launch_bounds__(RS_THREADS) k_rs_scatter(
    const unsigned long long* __restrict__ keys, const uint32_t* __restrict__ vals, size_t n,
    int shift, const uint32_t* __restrict__ offsets, uint32_t ntiles,
    unsigned long long* __restrict__ keys_out, uint32_t* __restrict__ vals_out) {
    // VALS = false: keys-only (packed) sort -- no value registers or staging,
    // so more CTAs fit per SM to hide the key-load latency
    constexpr int RADIX = 1 << BITS;
    constexpr int DPT = RADIX / RS_THREADS;       // digits per thread (1 or 2)
    static_assert(DPT >= 1 && RADIX % RS_THREADS == 0, "RADIX must be a multiple of the CTA");
    __shared__ uint32_t wcnt[RS_WARPS][RADIX + 1];
    __shared__ uint32_t tile_base[RADIX];
    __shared__ uint32_t local_off[RADIX];
    __shared__ uint32_t warp_tot[RS_WARPS];
    __shared__ unsigned long long sk[RS_TILE];
    __shared__ uint32_t sv[VALS ? RS_TILE : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int j = lane; j < RADIX + 1; j += 32) wcnt[warp][j] = 0;
    for (int j = threadIdx.x; j < RADIX; j += RS_THREADS)
        tile_base[j] = offsets[(size_t)j * ntiles + blockIdx.x];
    __syncwarp();

    const size_t wbase = (size_t)blockIdx.x * RS_TILE + (size_t)warp * (32 * RS_ITEMS);
    unsigned long long k[RS_ITEMS];
    uint32_t v[RS_ITEMS], dig[RS_ITEMS], rank[RS_ITEMS];
#pragma unroll
    for (int i = 0; i < RS_ITEMS; ++i) {
        size_t idx = wbase + (size_t)i * 32 + lane;
        bool ok = idx < n;
        k[i] = ok ? keys[idx] : 0ull;
        v[i] = (VALS && ok) ? vals[idx] : 0u;
        dig[i] = ok ? ((uint32_t)(k[i] >> shift) & (RADIX - 1)) : (uint32_t)RADIX;
    }
    const uint32_t lt_mask = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < RS_ITEMS; ++i) {
        // lanes holding the same digit: BITS ballots (warp multi-split); the
        // match.any instruction it replaces was the kernel's bottleneck
        // (ncu: 33% of stall samples waiting on it)
        uint32_t peers = __ballot_sync(0xffffffffu, dig[i] < (uint32_t)RADIX);
#pragma unroll
        for (int b = 0; b < BITS; ++b) {
            const uint32_t bal = __ballot_sync(0xffffffffu, (dig[i] >> b) & 1u);
            peers &= ((dig[i] >> b) & 1u) ? bal : ~bal;
        }
        if (dig[i] >= (uint32_t)RADIX) peers = 1u << lane;   // sentinel lanes: alone
        int leader = __ffs(peers) - 1;
        uint32_t old = 0;
        if (lane == leader && dig[i] < (uint32_t)RADIX) {
            old = wcnt[warp][dig[i]];
            wcnt[warp][dig[i]] = old + __popc(peers);
        }
        old = __shfl_sync(0xffffffffu, old, leader);
        rank[i] = old + __popc(peers & lt_mask);
        __syncwarp();
    }
    __syncthreads();
    // cross-warp prefix per digit; this thread owns digits [t*DPT, t*DPT+DPT)
    uint32_t tile_count[DPT];
    uint32_t my_total = 0;
#pragma unroll
    for (int j = 0; j < DPT; ++j) {
        const int dgt = threadIdx.x * DPT + j;
        uint32_t run = 0;
#pragma unroll
        for (int w = 0; w < RS_WARPS; ++w) {
            uint32_t c = wcnt[w][dgt];
            wcnt[w][dgt] = run;
            run += c;
        }
        tile_count[j] = run;
        my_total += run;
    }
    // tile-local digit offsets (exclusive scan of the tile histogram)
    {
        uint32_t inc = my_total;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        if (lane == 31) warp_tot[warp] = inc;
        __syncthreads();
        uint32_t pre = 0;
        for (int w = 0; w < warp; ++w) pre += warp_tot[w];
        uint32_t run = pre + inc - my_total;
#pragma unroll
        for (int j = 0; j < DPT; ++j) {
            local_off[threadIdx.x * DPT + j] = run;
            run += tile_count[j];
        }
    }
    __syncthreads();
    // stage the tile in digit order in shared memory ...
#pragma unroll
    for (int i = 0; i < RS_ITEMS; ++i) {
        if (dig[i] < (uint32_t)RADIX) {
            const uint32_t lpos = local_off[dig[i]] + wcnt[warp][dig[i]] + rank[i];
            sk[lpos] = k[i];
            if (VALS) sv[lpos] = v[i];
        }
    }
    __syncthreads();
    // ... then write it out with consecutive threads on consecutive positions
    // of each digit's output run (coalesced instead of 32 scattered lines)
    const size_t tbase = (size_t)blockIdx.x * RS_TILE;
    const uint32_t tn = (uint32_t)min((size_t)RS_TILE, n - tbase);
    for (uint32_t i = threadIdx.x; i < tn; i += RS_THREADS) {
        const unsigned long long key = sk[i];
        const uint32_t dg = (uint32_t)(key >> shift) & (RADIX - 1);
        const uint32_t dst = tile_base[dg] + (i - local_off[dg]);
        keys_out[dst] = key;
        if (VALS) vals_out[dst] = sv[i];
    }
}

// ------------------------------------------------------------ onesweep
// One kernel per 8-bit pass.  Tiles take their ids in launch order from an
// atomic counter, rank their keys as k_rs_scatter does, publish their digit
// counts and find their global offsets by decoupled look-back over the
// preceding tiles' published counts; the digit bases come from one histogram
// of all passes computed up front (k_rs_hist_all, or fused into the kernel
// that produced the keys).  A pass then reads and writes the keys once,
// where hist + scan + scatter reads them twice and adds two launches.
constexpr int OS_ITEMS = 12;
constexpr int OS_TILE = RS_THREADS * OS_ITEMS;    // 3072 keys per tile
constexpr uint32_t OS_AGG = 1u << 30;             // status word: count of this tile only
constexpr uint32_t OS_PRE = 2u << 30;             // status word: inclusive prefix
constexpr uint32_t OS_VAL = OS_AGG - 1u;
constexpr int OS_LB = 8;                          // look-back window

__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Digit histograms of all passes in one read of the keys (caller zeroes hist).
__global__ void __launch_bounds__(RS_THREADS) k_rs_hist_all(const unsigned long long* __restrict__ keys,
                                                            size_t n, const PassPlan plan,
                                                            uint32_t* __restrict__ hist) {
    __shared__ uint32_t h[OS_MAXPASS * OS_HSTRIDE];
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += RS_THREADS) h[j] = 0;
    __syncthreads();
    for (size_t i = (size_t)blockIdx.x * RS_THREADS + threadIdx.x; i < n;
         i += (size_t)gridDim.x * RS_THREADS) {
        const unsigned long long k = keys[i];
        for (int p = 0; p < plan.npass; ++p)
            atomicAdd(&h[p * OS_HSTRIDE + ((k >> plan.shift[p]) & ((1u << plan.bits[p]) - 1u))], 1u);
    }
    __syncthreads();
    for (int j = threadIdx.x; j < plan.npass * OS_HSTRIDE; j += RS_THREADS)
        if (h[j]) atomicAdd(hist + j, h[j]);
}

// Exclusive scan of each pass's (up to 512) digit counts, in place (one CTA
// per pass, two digits per thread).
__global__ void __launch_bounds__(RS_THREADS) k_rs_hist_scan(uint32_t* __restrict__ hist) {
    uint32_t* h = hist + (size_t)blockIdx.x * OS_HSTRIDE;
    const uint32_t c0 = h[2 * threadIdx.x], c1 = h[2 * threadIdx.x + 1];
    uint32_t total;
    const uint32_t ex = block_exclusive_scan<uint32_t>(c0 + c1, &total);
    h[2 * threadIdx.x] = ex;
    h[2 * threadIdx.x + 1] = ex + c0;
}

// One pass over a digit of RB bits (8: 256 digits, one per thread; 9: 512,
// two per thread -- a 34-bit key then takes 9+9+8+8 instead of five 8-bit
// passes).
template <bool VALS, int MINB, int RB, int ITEMS = OS_ITEMS, int LB = OS_LB>
__global__ void __launch_bounds__(RS_THREADS, MINB) k_onesweep(
    const unsigned long long* __restrict__ keys, const uint32_t* __restrict__ vals, size_t n,
    int shift, const uint32_t* __restrict__ gbase, uint32_t* status, uint32_t* tile_ctr,
    unsigned long long* __restrict__ keys_out, uint32_t* __restrict__ vals_out,
    uint32_t sleep_ns, uint32_t* __restrict__ rows_out, unsigned long long row_mask) {
    constexpr int RADIX = 1 << RB;
    constexpr int TILE = RS_THREADS * ITEMS;
    constexpr int DPT = RADIX / RS_THREADS;          // digits per thread
    static_assert(DPT == 1 || DPT == 2, "8- or 9-bit digits");
    constexpr uint32_t DMASK = RADIX - 1;
    constexpr int RSH = RB + 1;                      // rank shift in dr (digit RADIX = sentinel)
    __shared__ uint32_t wcnt[RS_WARPS][RADIX + 1];
    __shared__ uint32_t tile_base[RADIX];
    __shared__ uint32_t local_off[RADIX];
    __shared__ uint32_t warp_tot[RS_WARPS];
    __shared__ uint32_t s_tile;
    __shared__ unsigned long long sk[TILE];
    __shared__ uint32_t sv[VALS ? TILE : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
    for (int j = lane; j < RADIX + 1; j += 32) wcnt[warp][j] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;

    // ---- load and rank (warp w owns a contiguous chunk of 32 * ITEMS keys)
    const size_t wbase = (size_t)tile * TILE + (size_t)warp * (32 * ITEMS);
    unsigned long long k[ITEMS];
    uint32_t v[VALS ? ITEMS : 1];
    uint32_t dr[ITEMS];                       // digit | rank << RSH; digit RADIX: past the end
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        const size_t idx = wbase + (size_t)i * 32 + lane;
        const bool ok = idx < n;
        k[i] = ok ? keys[idx] : 0ull;
        if (VALS) v[i] = ok ? vals[idx] : 0u;
        dr[i] = ok ? ((uint32_t)(k[i] >> shift) & DMASK) : (uint32_t)RADIX;
    }
    const uint32_t lt_mask = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        const uint32_t dig = dr[i];
        uint32_t peers = __ballot_sync(0xffffffffu, dig < (uint32_t)RADIX);
#pragma unroll
        for (int b = 0; b < RB; ++b) {
            const uint32_t bal = __ballot_sync(0xffffffffu, (dig >> b) & 1u);
            peers &= ((dig >> b) & 1u) ? bal : ~bal;
        }
        if (dig >= (uint32_t)RADIX) peers = 1u << lane;
        // the group's highest lane updates the counter: its rank below is
        // the group size - 1 (one popc and one clz per key)
        const uint32_t below = __popc(peers & lt_mask);
        const int leader = 31 - __clz(peers);
        uint32_t old = 0;
        if (lane == leader && dig < (uint32_t)RADIX) {
            old = wcnt[warp][dig];
            wcnt[warp][dig] = old + below + 1u;
        }
        old = __shfl_sync(0xffffffffu, old, leader);
        dr[i] = dig | ((old + below) << RSH);
        __syncwarp();
    }
    __syncthreads();

    // ---- thread t owns digits t*DPT .. t*DPT+DPT-1: cross-warp prefix, look-back
    const int t = threadIdx.x;
    uint32_t count[DPT], excl[DPT];
#pragma unroll
    for (int c = 0; c < DPT; ++c) {
        const int dg = t * DPT + c;
        uint32_t acc = 0;
#pragma unroll
        for (int w = 0; w < RS_WARPS; ++w) {
            const uint32_t x = wcnt[w][dg];
            wcnt[w][dg] = acc;
            acc += x;
        }
        count[c] = acc;
        excl[c] = 0;
    }
    uint32_t* mine = status + (size_t)tile * RADIX + t * DPT;
    if (tile == 0) {
#pragma unroll
        for (int c = 0; c < DPT; ++c) st_relaxed(mine + c, OS_PRE | count[c]);
    } else {
#pragma unroll
        for (int c = 0; c < DPT; ++c) st_relaxed(mine + c, OS_AGG | count[c]);
        // windowed look-back: LB predecessors per round trip (in the first
        // wave every tile has only aggregates behind it; one tile per round
        // trip would serialise the wave)
#pragma unroll
        for (int c = 0; c < DPT; ++c) {
            int32_t j = (int32_t)tile - 1;          // next predecessor to account for
            bool done = false;
            while (!done) {
                uint32_t w[LB];
#pragma unroll
                for (int q = 0; q < LB; ++q)
                    w[q] = j - q >= 0 ? ld_relaxed(status + (size_t)(j - q) * RADIX + t * DPT + c)
                                      : OS_PRE;
                bool wait = false;
#pragma unroll
                for (int q = 0; q < LB; ++q) {
                    if (done || wait) break;
                    if (w[q] == 0u) {                // not published yet: poll again from j
                        wait = true;
                        break;
                    }
                    excl[c] += w[q] & OS_VAL;
                    --j;
                    if (w[q] & OS_PRE) done = true;
                }
                // back off instead of spinning: polling loads and branches
                // would take issue slots from the other CTAs' ranking and scatter
                if (wait && sleep_ns) __nanosleep(sleep_ns);
            }
            st_relaxed(mine + c, OS_PRE | (excl[c] + count[c]));
        }
    }
#pragma unroll
    for (int c = 0; c < DPT; ++c) tile_base[t * DPT + c] = gbase[t * DPT + c] + excl[c];
    {   // tile-local digit offsets
        uint32_t tc = 0;
#pragma unroll
        for (int c = 0; c < DPT; ++c) tc += count[c];
        uint32_t inc = tc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        if (lane == 31) warp_tot[warp] = inc;
        __syncthreads();
        uint32_t pre = 0;
        for (int w = 0; w < warp; ++w) pre += warp_tot[w];
        pre += inc - tc;
#pragma unroll
        for (int c = 0; c < DPT; ++c) {
            local_off[t * DPT + c] = pre;
            pre += count[c];
        }
    }
    __syncthreads();
    // ---- stage in digit order, write out coalesced
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        const uint32_t dig = dr[i] & ((2u << RB) - 1u);
        if (dig < (uint32_t)RADIX) {
            const uint32_t lpos = local_off[dig] + wcnt[warp][dig] + (dr[i] >> RSH);
            sk[lpos] = k[i];
            if (VALS) sv[lpos] = v[i];
        }
    }
    __syncthreads();
    const size_t tbase = (size_t)tile * TILE;
    const uint32_t tn = (uint32_t)min((size_t)TILE, n - tbase);
    for (uint32_t i = threadIdx.x; i < tn; i += RS_THREADS) {
        const unsigned long long key = sk[i];
        const uint32_t dg = (uint32_t)(key >> shift) & DMASK;
        const uint32_t dst = tile_base[dg] + (i - local_off[dg]);
        if (rows_out) rows_out[dst] = (uint32_t)(key & row_mask);   // last pass: rows only
        else keys_out[dst] = key;
        if (VALS) vals_out[dst] = sv[i];
    }
}

bool onesweep_enabled(size_t n) {
    static const bool on = [] {                  // DTS_ONESWEEP=0: hist + scan + scatter
        const char* e = getenv("DTS_ONESWEEP");
        return !(e && e[0] == '0');
    }();
    return on && n < (size_t)OS_VAL;
}

// Digit plan for key bits [lo, hi): as few passes as 9-bit digits allow,
// 8-bit digits where they suffice (DTS_RADIX9=0: 8-bit digits only; key +
// value sorts keep 8-bit digits: a 9-bit tile with values exceeds 48 KB).
}  // namespace

PassPlan plan_passes(int lo, int hi, bool allow9) {
    static const bool r9 = [] {
        const char* e = getenv("DTS_RADIX9");
        return !(e && e[0] == '0');
    }();
    const int nb = hi - lo;
    int np = (nb + 7) / 8;
    int n9 = 0;
    if (r9 && allow9 && np > 1 && nb <= 9 * (np - 1)) {
        --np;
        n9 = nb - 8 * np;                      // passes that need a 9th bit
    }
    PassPlan pl{};
    pl.npass = np;
    int sh = lo;
    for (int p = 0; p < np; ++p) {
        pl.bits[p] = p < n9 ? 9 : 8;
        pl.shift[p] = sh;
        sh += pl.bits[p];
    }
    return pl;
}

namespace {
template <bool VALS, int MINB, int RB, int ITEMS = OS_ITEMS>
void launch_onesweep(uint32_t ntiles, cudaStream_t s, const unsigned long long* kin,
                     const uint32_t* vin, size_t n, int shift, const uint32_t* gbase,
                     uint32_t* status, uint32_t* ctr, unsigned long long* kout, uint32_t* vout,
                     uint32_t sleep_ns, uint32_t* rows_out = nullptr,
                     unsigned long long row_mask = 0) {
    k_onesweep<VALS, MINB, RB, ITEMS><<<ntiles, RS_THREADS, 0, s>>>(kin, vin, n, shift, gbase,
                                                                    status, ctr, kout, vout,
                                                                    sleep_ns, rows_out, row_mask);
}

// Keys-only tile shapes (DTS_OS_SHAPE, A/B): 0 = 12 keys per thread for
// both digit widths (3072-key tiles); 1 (default) = 16 (8-bit, 3 CTAs/SM)
// and 13 (9-bit); 2 = 16 (8-bit, 4 CTAs/SM, spills) and 13 (9-bit).
// Measured on the C4 entry sort (9+9+8+8): 0.834, 0.817, 0.828 ms.
int os_shape() {
    static const int v = [] {
        const char* e = getenv("DTS_OS_SHAPE");
        return e ? atoi(e) : 1;
    }();
    return v;
}
int os_items(int bits, bool vals) {
    if (vals || os_shape() == 0) return OS_ITEMS;
    return bits == 9 ? 13 : 16;
}

// The plan's onesweep passes; hist holds each pass's exclusive digit bases
// (k_rs_hist_scan).  On return *kin / *vin hold the result.
void onesweep_passes(unsigned long long** kin, unsigned long long** kout, uint32_t** vin,
                     uint32_t** vout, size_t n, const PassPlan& plan, const uint32_t* hist,
                     cudaStream_t s, uint32_t* rows_out = nullptr,
                     unsigned long long row_mask = 0) {
    uint32_t maxtiles = 0;
    for (int p = 0; p < plan.npass; ++p) {
        const uint32_t tile = RS_THREADS * os_items(plan.bits[p], *vin != nullptr);
        maxtiles = std::max(maxtiles, (uint32_t)((n + tile - 1) / tile));
    }
    const size_t nstat = (size_t)maxtiles * OS_HSTRIDE + 32;
    DevBuf<uint32_t> status(nstat, s);
    static const uint32_t sleep_ns = [] {   // DTS_OS_SLEEP: look-back back-off (ns)
        const char* e = getenv("DTS_OS_SLEEP");   // C4 entry sort, 5 passes: 0 ns
        return e ? (uint32_t)atoi(e) : 256u;      // 0.984 ms, 32: 0.970, 128: 0.961,
    }();                                          // 512: 0.957 (look-back window 8:
                                                  // 0.936, 16: 1.03, 32: 1.64)
    for (int p = 0; p < plan.npass; ++p) {
        const uint32_t tile = RS_THREADS * os_items(plan.bits[p], *vin != nullptr);
        const uint32_t ntiles = (uint32_t)((n + tile - 1) / tile);
        const int shape = *vin ? 0 : os_shape();
        const size_t used = (size_t)ntiles << plan.bits[p];
        DTS_CUDA(cudaMemsetAsync(status.p, 0, (used + 32) * sizeof(uint32_t), s));
        uint32_t* ctr = status.p + used;
        const uint32_t* gb = hist + OS_HSTRIDE * p;
        const int sh = plan.shift[p];
        uint32_t* ro = (p == plan.npass - 1 && !*vin) ? rows_out : nullptr;
        if (plan.bits[p] == 9) {
            if (shape) launch_onesweep<false, 3, 9, 13>(ntiles, s, *kin, nullptr, n, sh, gb,
                                                        status.p, ctr, *kout, nullptr, sleep_ns, ro, row_mask);
            else launch_onesweep<false, 3, 9>(ntiles, s, *kin, nullptr, n, sh, gb, status.p, ctr,
                                              *kout, nullptr, sleep_ns, ro, row_mask);
        } else {
            if (*vin) launch_onesweep<true, 2, 8>(ntiles, s, *kin, *vin, n, sh, gb, status.p, ctr,
                                                  *kout, *vout, sleep_ns);
            else if (shape == 1)
                launch_onesweep<false, 3, 8, 16>(ntiles, s, *kin, nullptr, n, sh, gb, status.p,
                                                 ctr, *kout, nullptr, sleep_ns, ro, row_mask);
            else if (shape == 2)
                launch_onesweep<false, 4, 8, 16>(ntiles, s, *kin, nullptr, n, sh, gb, status.p,
                                                 ctr, *kout, nullptr, sleep_ns, ro, row_mask);
            else launch_onesweep<false, 4, 8>(ntiles, s, *kin, nullptr, n, sh, gb, status.p, ctr,
                                              *kout, nullptr, sleep_ns, ro, row_mask);
        }
        DTS_LAUNCH_CHECK();
        std::swap(*kin, *kout);
        std::swap(*vin, *vout);
    }
}

template <int BITS>
void radix_pass(const unsigned long long* kin, const uint32_t* vin, unsigned long long* kout,
                uint32_t* vout, size_t n, int shift, uint32_t ntiles, uint32_t* counts,
                uint32_t* offs, cudaStream_t s) {
    const size_t ncount = ((size_t)1 << BITS) * ntiles;
    k_rs_hist<BITS><<<ntiles, RS_THREADS, 0, s>>>(kin, n, shift, counts, ntiles);
    DTS_LAUNCH_CHECK();
    scan_exclusive_u32_to_u32(counts, offs, ncount, s);
    if (vin)
        k_rs_scatter<BITS, true><<<ntiles, RS_THREADS, 0, s>>>(kin, vin, n, shift, offs, ntiles,
                                                               kout, vout);
    else
        k_rs_scatter<BITS, false><<<ntiles, RS_THREADS, 0, s>>>(kin, vin, n, shift, offs, ntiles,
                                                                kout, vout);
    DTS_LAUNCH_CHECK();
}
}  // namespace

unsigned long long* radix_sort_keys_hist(unsigned long long* keys, unsigned long long* tmp,
                                         size_t n, const PassPlan& plan, uint32_t* hist,
                                         cudaStream_t s, uint32_t* rows_out,
                                         unsigned long long row_mask) {
    k_rs_hist_scan<<<plan.npass, RS_THREADS, 0, s>>>(hist);
    DTS_LAUNCH_CHECK();
    unsigned long long *kin = keys, *kout = tmp;
    uint32_t *vin = nullptr, *vout = nullptr;
    onesweep_passes(&kin, &kout, &vin, &vout, n, plan, hist, s, rows_out, row_mask);
    return rows_out ? nullptr : kin;
}

bool radix_onesweep(size_t n) { return onesweep_enabled(n); }

unsigned long long* radix_sort_keys(unsigned long long* keys, unsigned long long* tmp, size_t n,
                                    int lo, int hi, cudaStream_t s) {
    if (n <= 1 || hi <= lo) return keys;
    if (onesweep_enabled(n)) {
        const PassPlan plan = plan_passes(lo, hi, true);
        DevBuf<uint32_t> hist((size_t)plan.npass * OS_HSTRIDE, s);
        DTS_CUDA(cudaMemsetAsync(hist.p, 0, (size_t)plan.npass * OS_HSTRIDE * sizeof(uint32_t), s));
        const unsigned hb = (unsigned)std::min<size_t>((n + RS_THREADS - 1) / RS_THREADS, 148 * 8);
        k_rs_hist_all<<<hb, RS_THREADS, 0, s>>>(keys, n, plan, hist.p);
        DTS_LAUNCH_CHECK();
        k_rs_hist_scan<<<plan.npass, RS_THREADS, 0, s>>>(hist.p);
        DTS_LAUNCH_CHECK();
        unsigned long long *kin = keys, *kout = tmp;
        uint32_t *vin = nullptr, *vout = nullptr;
        onesweep_passes(&kin, &kout, &vin, &vout, n, plan, hist.p, s);
        return kin;
    }
    const uint32_t ntiles = (uint32_t)((n + RS_TILE - 1) / RS_TILE);
    const size_t ncount = (size_t)256 * ntiles;
    DevBuf<uint32_t> counts(ncount, s), offs(ncount + 1, s);
    unsigned long long *kin = keys, *kout = tmp;
    for (int shift = lo; shift < hi; shift += 8) {
        radix_pass<8>(kin, nullptr, kout, nullptr, n, shift, ntiles, counts.p, offs.p, s);
        unsigned long long* t = kin;
        kin = kout;
        kout = t;
    }
    return kin;
}

void radix_sort_pairs(unsigned long long* keys, uint32_t* vals, unsigned long long* keys_tmp,
                      uint32_t* vals_tmp, size_t n, int nbits, cudaStream_t s) {
    if (n <= 1 || nbits <= 0) return;
    if (onesweep_enabled(n)) {
        const PassPlan plan = plan_passes(0, nbits, false);
        const int npass = plan.npass;
        DevBuf<uint32_t> hist((size_t)npass * OS_HSTRIDE, s);
        DTS_CUDA(cudaMemsetAsync(hist.p, 0, (size_t)npass * OS_HSTRIDE * sizeof(uint32_t), s));
        const unsigned hb = (unsigned)std::min<size_t>((n + RS_THREADS - 1) / RS_THREADS, 148 * 8);
        k_rs_hist_all<<<hb, RS_THREADS, 0, s>>>(keys, n, plan, hist.p);
        DTS_LAUNCH_CHECK();
        k_rs_hist_scan<<<npass, RS_THREADS, 0, s>>>(hist.p);
        DTS_LAUNCH_CHECK();
        unsigned long long *kin = keys, *kout = keys_tmp;
        uint32_t *vin = vals, *vout = vals_tmp;
        onesweep_passes(&kin, &kout, &vin, &vout, n, plan, hist.p, s);
        if (npass & 1) {
            DTS_CUDA(cudaMemcpyAsync(keys, kin, n * sizeof(unsigned long long),
                                     cudaMemcpyDeviceToDevice, s));
            DTS_CUDA(cudaMemcpyAsync(vals, vin, n * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
        }
        return;
    }
    // 8-bit digits: measured on C4 (35-bit keys) the 9-bit variant's 4 passes
    // cost more than 5 8-bit passes (45 KB of shared memory per CTA lowers
    // occupancy; 113 vs 80 us per pass at 20 M keys).  DTS_RADIX_BITS=9 opts in.
    static const int pref = [] {
        const char* e = getenv("DTS_RADIX_BITS");
        return (e && atoi(e) == 9) ? 9 : 8;
    }();
    const int bits = (pref == 9 && (nbits + 8) / 9 < (nbits + 7) / 8) ? 9 : 8;
    const uint32_t ntiles = (uint32_t)((n + RS_TILE - 1) / RS_TILE);
    const size_t ncount = ((size_t)1 << bits) * ntiles;
    DevBuf<uint32_t> counts(ncount, s), offs(ncount + 1, s);
    unsigned long long *kin = keys, *kout = keys_tmp;
    uint32_t *vin = vals, *vout = vals_tmp;
    int passes = 0;
    for (int shift = 0; shift < nbits; shift += bits, ++passes) {
        if (bits == 9) radix_pass<9>(kin, vin, kout, vout, n, shift, ntiles, counts.p, offs.p, s);
        else radix_pass<8>(kin, vin, kout, vout, n, shift, ntiles, counts.p, offs.p, s);
        unsigned long long* tk = kin; kin = kout; kout = tk;
        uint32_t* tv = vin; vin = vout; vout = tv;
    }
    if (passes & 1) {
        DTS_CUDA(cudaMemcpyAsync(keys, kin, n * sizeof(unsigned long long),
                                 cudaMemcpyDeviceToDevice, s));
        DTS_CUDA(cudaMemcpyAsync(vals, vin, n * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
    }
}

}  // namespace dts
