// api.cu -- the C ABI of include/dts.h: argument validation, device checks,
// host <-> device copies, ownership and error reporting.  Every step of the
// search itself runs in the kernels of build.cu / search.cu / prims.cu.
#include <cuda_runtime.h>

#include <sys/mman.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <string>
#include <condition_variable>
#include <exception>
#include <thread>
#include <vector>

#include "internal.cuh"

namespace dts {

std::atomic<unsigned long long> g_launches{0};
static thread_local std::string g_err;
void set_last_error(const std::string& msg) { g_err = msg; }

// Device memory of an index back to the device cache (alloc.cu): waits for
// the end of the build only (a build returns before its last kernels finish;
// searches are synchronous on return, so none is in flight), not for every
// stream of the device.
void free_index_arrays(dts_index* idx) {
    if (idx->ready) cudaEventSynchronize(idx->ready);
    for (int i = 0; i < idx->nev; ++i) cudaEventDestroy(idx->ev[i]);
    idx->nev = 0;
    idx->ready = nullptr;
    cache_free(idx->block);
    cache_free(idx->ht.slots);
    cache_free(idx->etraj);
    idx->etraj = nullptr;
    cache_free(idx->out_block);
    idx->out_block = nullptr;
    idx->out = dts::OutlierIndex{};
    for (int a = 0; a < 3; ++a) {
        cache_free(idx->sb_block[a]);
        idx->sb_block[a] = nullptr;
        cache_free(idx->sb_rec[a]);
        idx->sb_rec[a] = nullptr;
    }
    idx->block = nullptr;
    idx->ht.slots = nullptr;
}

namespace {

std::mutex g_mu;
bool g_pool_ready[64] = {false};

// Verify the device is an sm_100 part (the cubins are sm_100a-only) and make
// the stream-ordered pool keep its memory between calls.
void prepare_device(int dev) {
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        throw Error(DTS_ENOTSUP, "no CUDA device available");
    }
    if (dev < 0 || dev >= count) throw Error(DTS_EINVAL, "device ordinal out of range");
    DTS_CUDA(cudaSetDevice(dev));
    std::lock_guard<std::mutex> lk(g_mu);
    if (dev < 64 && !g_pool_ready[dev]) {
        cudaDeviceProp prop;
        DTS_CUDA(cudaGetDeviceProperties(&prop, dev));
        if (prop.major != 10 || prop.minor != 0)
            throw Error(DTS_ENOTSUP, std::string("libdts is built for sm_100a; device is ") +
                                         prop.name + " sm_" + std::to_string(prop.major) +
                                         std::to_string(prop.minor));
        cudaMemPool_t pool;
        DTS_CUDA(cudaDeviceGetDefaultMemPool(&pool, dev));
        unsigned long long thr = ~0ull;
        DTS_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
        g_pool_ready[dev] = true;
    }
}

// Pinned host result blocks, recycled (the result D2H is part of the
// search response time; cudaMallocHost per call would dominate it).
constexpr size_t HDR = 64;
std::multimap<size_t, void*> g_pinned_free;
size_t g_pinned_cached = 0;

void* pinned_alloc(size_t bytes) {
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_pinned_free.lower_bound(bytes);
        if (it != g_pinned_free.end() && it->first <= 2 * bytes + (1u << 20)) {
            void* b = it->second;
            g_pinned_cached -= it->first;
            g_pinned_free.erase(it);
            return static_cast<char*>(b) + HDR;
        }
    }
    void* b = nullptr;
    // large outputs use pageable memory: page-locking gigabytes costs far more
    // (measured ~0.7 s/GB) than the driver-staged copy it would speed up
    cudaError_t e = bytes <= (size_t(1) << 30) ? cudaMallocHost(&b, bytes + HDR)
                                               : cudaErrorMemoryAllocation;
    size_t kind = 0;
    if (e != cudaSuccess) {
        cudaGetLastError();
        // 2 MiB aligned and backed by transparent huge pages where the
        // kernel allows: first-touch faults of a 10 GB result array at 4 KiB
        // granularity cost more than its PCIe transfer
        if (posix_memalign(&b, size_t(2) << 20, bytes + HDR) != 0) b = nullptr;
        if (!b) throw Error(DTS_ENOMEM, "host allocation failed for the result buffer");
        madvise(b, bytes + HDR, MADV_HUGEPAGE);
        kind = 1;
    }
    static_cast<size_t*>(b)[0] = bytes;
    static_cast<size_t*>(b)[1] = kind;
    return static_cast<char*>(b) + HDR;
}

bool is_pageable_block(const void* p) {
    const void* b = static_cast<const char*>(p) - HDR;
    return static_cast<const size_t*>(b)[1] == 1;
}

// Device -> host copy of `bytes` into (part of) a result block of
// pinned_alloc (`pageable`: is_pageable_block of that block).  A pinned
// block takes one cudaMemcpyAsync; a pageable one (outputs over
// 1 GB) is staged through two pinned 64 MiB buffers of the calling thread:
// the DMA of chunk i runs while host threads copy chunk i-1 out (and take
// the destination's first-touch page faults in parallel) -- a single
// driver-staged copy into pageable memory runs at the speed of one core.
void copy_results_d2h(void* dst, const void* src, size_t bytes, cudaStream_t s, bool pageable) {
    if (!bytes) return;
    if (!pageable || bytes < (size_t(256) << 20)) {
        DTS_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
        return;
    }
    constexpr size_t CH = size_t(64) << 20;
    struct Stage {
        void* buf[2] = {nullptr, nullptr};
        cudaEvent_t ev[2] = {nullptr, nullptr};
        ~Stage() {                                // thread exit (stream workers)
            for (int i = 0; i < 2; ++i) {
                if (buf[i]) cudaFreeHost(buf[i]);
                if (ev[i]) cudaEventDestroy(ev[i]);
            }
        }
    };
    static thread_local Stage st;
    if (!st.buf[0]) {
        for (int i = 0; i < 2; ++i) {
            DTS_CUDA(cudaMallocHost(&st.buf[i], CH));
            DTS_CUDA(cudaEventCreateWithFlags(&st.ev[i], cudaEventDisableTiming));
        }
    }
    const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
    const unsigned nt = std::min(8u, hw);
    auto host_copy = [&](char* d, const char* p, size_t n) {
        std::vector<std::thread> th;
        const size_t per = (n + nt - 1) / nt;
        for (unsigned t = 1; t < nt; ++t) {
            const size_t a = std::min(n, t * per), b = std::min(n, a + per);
            if (a < b) th.emplace_back([=] { std::memcpy(d + a, p + a, b - a); });
        }
        std::memcpy(d, p, std::min(n, per));
        for (auto& x : th) x.join();
    };
    const size_t nch = (bytes + CH - 1) / CH;
    for (size_t i = 0; i <= nch; ++i) {
        if (i < nch) {
            const size_t off = i * CH, n = std::min(CH, bytes - off);
            DTS_CUDA(cudaMemcpyAsync(st.buf[i & 1], static_cast<const char*>(src) + off, n,
                                     cudaMemcpyDeviceToHost, s));
            DTS_CUDA(cudaEventRecord(st.ev[i & 1], s));
        }
        if (i > 0) {
            const size_t j = i - 1, off = j * CH, n = std::min(CH, bytes - off);
            DTS_CUDA(cudaEventSynchronize(st.ev[j & 1]));
            host_copy(static_cast<char*>(dst) + off, static_cast<const char*>(st.buf[j & 1]), n);
        }
    }
}

void pinned_free(void* p) {
    if (!p) return;
    void* b = static_cast<char*>(p) - HDR;
    size_t bytes = static_cast<size_t*>(b)[0];
    if (static_cast<size_t*>(b)[1] == 1) {
        std::free(b);
        return;
    }
    std::lock_guard<std::mutex> lk(g_mu);
    if (g_pinned_cached + bytes <= (size_t(4) << 30)) {
        g_pinned_free.emplace(bytes, b);
        g_pinned_cached += bytes;
    } else {
        cudaFreeHost(b);
    }
}

void free_index_memory(dts_index* idx) {
    if (!idx) return;
    DeviceGuard dg;
    cudaSetDevice(idx->device);
    free_index_arrays(idx);
    ooc_free(idx->ooc);
    idx->ooc = nullptr;
}

dts_index_params defaults() {
    dts_index_params p{};
    return p;
}

void check_params(const dts_index_params& p) {
    if (!(p.d_hint >= 0.0) || !std::isfinite(p.d_hint))
        throw Error(DTS_EINVAL, "d_hint must be finite and >= 0");
    if (p.method > DTS_METHOD_SUBBIN) throw Error(DTS_EINVAL, "unknown method");
}

void check_aligned(const void* p, const char* what) {
    if (reinterpret_cast<uintptr_t>(p) & 15u)
        throw Error(DTS_EINVAL, std::string(what) + " must be 16-byte aligned");
}

template <typename F>
dts_status guarded(F&& f) {
    try {
        g_err.clear();
        f();
        return DTS_OK;
    } catch (const Error& e) {
        g_err = e.what();
        return e.status;
    } catch (const std::bad_alloc&) {
        g_err = "host allocation failed";
        return DTS_ENOMEM;
    } catch (const std::exception& e) {
        g_err = e.what();
        return DTS_EINTERNAL;
    } catch (...) {
        g_err = "unknown internal error";
        return DTS_EINTERNAL;
    }
}

dts_status build_common(const dts_segment* D, size_t n, const dts_index_params* params,
                        bool host, cudaStream_t s, dts_index** out_index) {
    if (out_index) *out_index = nullptr;
    dts_index* idx = nullptr;
    DeviceGuard dg;
    dts_status st = guarded([&] {
        if (!out_index) throw Error(DTS_EINVAL, "out_index is NULL");
        if (n > 0 && !D) throw Error(DTS_EINVAL, "D is NULL with n > 0");
        if (n >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "n must be < 2^32");
        dts_index_params p = params ? *params : defaults();
        check_params(p);
        prepare_device(p.device);
        idx = new dts_index();
        idx->device = p.device;
        if (n == 0) return;
        if (host && p.mem_budget_bytes && index_bytes_estimate(n) > p.mem_budget_bytes) {
            // D (and its index) exceed the budget: temporal shards in pinned
            // host memory, indexed one at a time at search time (ooc.cu)
            ooc_build(idx, D, n, p, s);
            DTS_CUDA(cudaStreamSynchronize(s));
            return;
        }
        if (host) {
            DevBuf<dts_segment> dD(n, s);
            DevBuf<uint32_t> dmap(p.entry_ids ? n : 0, s);
            DTS_CUDA(cudaMemcpyAsync(dD.p, D, n * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
            if (p.entry_ids) {
                DTS_CUDA(cudaMemcpyAsync(dmap.p, p.entry_ids, n * sizeof(uint32_t),
                                         cudaMemcpyHostToDevice, s));
                p.entry_ids = dmap.p;
            }
            DevBuf<uint32_t> dtraj(p.entry_traj ? n : 0, s);
            if (p.entry_traj) {
                DTS_CUDA(cudaMemcpyAsync(dtraj.p, p.entry_traj, n * sizeof(uint32_t),
                                         cudaMemcpyHostToDevice, s));
                p.entry_traj = dtraj.p;
            }
            build_index_device(idx, dD.p, n, p, s);
        } else {
            check_aligned(D, "D_dev");
            build_index_device(idx, D, n, p, s);
            return;                 // asynchronous on s after validation (dts.h)
        }
        DTS_CUDA(cudaStreamSynchronize(s));
    });
    if (st != DTS_OK) {
        if (idx) {
            free_index_memory(idx);
            delete idx;
        }
        return st;
    }
    *out_index = idx;
    return DTS_OK;
}

// Host-output search whose results exceed device memory: plan query-id
// chunks from the per-query counts so each chunk's results fit, search each
// chunk (ids offset by the chunk start) and copy its results to the host at
// the chunk's offset.  Concatenation in chunk order is the canonical order.
dts_result* search_streamed(const dts_index* index, const dts_segment* dQ, size_t nq, double d,
                            uint32_t qid_base, cudaStream_t s, const ResultsTooLarge& big,
                            dts_search_stats* stats, unsigned long long cap,
                            const uint32_t* qmap, const uint32_t* qtraj, bool excl) {
    size_t free_b = 0, total_b = 0;
    DTS_CUDA(cudaMemGetInfo(&free_b, &total_b));
    const unsigned long long budget = std::max<unsigned long long>(
        1, std::min<unsigned long long>(cap ? cap : ~0ull,
                                        (unsigned long long)(0.35 * (double)free_b / 72.0)));
    dts_result* h = static_cast<dts_result*>(pinned_alloc(big.total * sizeof(dts_result)));
    dts_search_stats agg{};
    if (stats) agg.time_kernels = stats->time_kernels;
    try {
        unsigned long long off = 0;
        size_t a = 0;
        while (a < nq) {
            size_t b = a;
            unsigned long long acc = 0;
            while (b < nq && (b == a || acc + big.counts[b] <= budget)) acc += big.counts[b++];
            SearchOut so;
            dts_search_stats cs{};
            search_device(index, dQ + a, b - a, d, qid_base + (uint32_t)a, s, &so, &cs, ~0ull,
                          qmap ? qmap + a : nullptr, qtraj ? qtraj + a : nullptr, excl);
            if (so.count != acc) {
                cache_free(so.results);
                throw Error(DTS_EINTERNAL, "streamed chunk count mismatch");
            }
            if (so.count) {
                copy_results_d2h(h + off, so.results, so.count * sizeof(dts_result), s,
                                 is_pageable_block(h));
                cache_free(so.results);
            }
            off += so.count;
            agg.candidates += cs.candidates;
            agg.cell_lookups += cs.cell_lookups;
            agg.max_results_per_query = std::max(agg.max_results_per_query,
                                                 cs.max_results_per_query);
            a = b;
        }
        agg.results = off;
    } catch (...) {
        pinned_free(h);
        throw;
    }
    if (stats) *stats = agg;
    return h;
}

// Host query set streamed through the device in chunks (
// the setting of the paper's prior work where Q does not fit on the GPU,
// P:L28): while chunk i is searched on the caller's stream, chunk i+1 is
// copied host -> device and the results of chunk i-1 device -> host on a
// copy stream, into one growing pinned output buffer.  Chunks are contiguous
// query-id ranges, so chunk-order concatenation is the canonical order.
dts_result* search_pipelined(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                             uint32_t qid_base, cudaStream_t s, size_t chunk,
                             const uint32_t* dmap, const uint32_t* dtraj, bool excl,
                             dts_search_stats* stats, size_t* out_count) {
    // H2D of chunk i+1 on cs and D2H of chunk i-1's results on ds run while
    // chunk i is searched on s: the two copy directions overlap (PCIe is
    // full duplex) and both overlap the search
    cudaStream_t cs = nullptr, ds = nullptr;
    DTS_CUDA(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    DTS_CUDA(cudaStreamCreateWithFlags(&ds, cudaStreamNonBlocking));
    cudaEvent_t h2d[2] = {nullptr, nullptr};
    struct Pending {
        dts_result* dev;
        size_t n;
    };
    std::vector<Pending> pending;
    dts_result* out = nullptr;
    size_t cap = 0, used = 0;
    dts_search_stats agg{};
    if (stats) agg.time_kernels = stats->time_kernels;
    auto cleanup = [&]() {
        if (cs) cudaStreamSynchronize(cs);
        if (ds) cudaStreamSynchronize(ds);
        for (auto& p : pending) cache_free(p.dev);
        pending.clear();
        for (auto& e : h2d) if (e) cudaEventDestroy(e);
        if (cs) cudaStreamDestroy(cs);
        if (ds) cudaStreamDestroy(ds);
        cs = ds = nullptr;
    };
    try {
        for (auto& e : h2d) DTS_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        DevBuf<dts_segment> qb0(chunk, s), qb1(chunk, s);
        dts_segment* qb[2] = {qb0.p, qb1.p};
        DTS_CUDA(cudaStreamSynchronize(s));          // buffers ready before the copy stream
        const size_t nchunks = (nq + chunk - 1) / chunk;
        auto issue_h2d = [&](size_t i) {
            const size_t a = i * chunk, m = std::min(chunk, nq - a);
            DTS_CUDA(cudaMemcpyAsync(qb[i & 1], Q + a, m * sizeof(dts_segment),
                                     cudaMemcpyHostToDevice, cs));
            DTS_CUDA(cudaEventRecord(h2d[i & 1], cs));
        };
        issue_h2d(0);
        for (size_t i = 0; i < nchunks; ++i) {
            const size_t a = i * chunk, m = std::min(chunk, nq - a);
            DTS_CUDA(cudaStreamWaitEvent(s, h2d[i & 1], 0));
            if (i + 1 < nchunks) issue_h2d(i + 1);   // buffer (i+1)&1 is free: search i-1 done
            SearchOut so;
            dts_search_stats cs_stats{};
            cs_stats.time_kernels = agg.time_kernels;
            search_device(index, qb[i & 1], m, d, qid_base + (uint32_t)a, s, &so, &cs_stats,
                          ~0ull, dmap ? dmap + a : nullptr, dtraj ? dtraj + a : nullptr, excl);
            if (so.count) {
                if (used + so.count > cap) {          // grow the pinned output
                    DTS_CUDA(cudaStreamSynchronize(ds));
                    const size_t want = std::max(used + so.count,
                                                 (size_t)((double)(used + so.count) *
                                                          (double)nchunks / (double)(i + 1) * 1.2));
                    dts_result* bigger = static_cast<dts_result*>(
                        pinned_alloc(want * sizeof(dts_result)));
                    if (used) std::memcpy(bigger, out, used * sizeof(dts_result));
                    pinned_free(out);
                    out = bigger;
                    cap = want;
                }
                DTS_CUDA(cudaMemcpyAsync(out + used, so.results, so.count * sizeof(dts_result),
                                         cudaMemcpyDeviceToHost, ds));
                pending.push_back({so.results, so.count});
                used += so.count;
            }
            agg.candidates += cs_stats.candidates;
            agg.cell_lookups += cs_stats.cell_lookups;
            agg.max_results_per_query =
                std::max(agg.max_results_per_query, cs_stats.max_results_per_query);
            agg.ms_prep += cs_stats.ms_prep;
            agg.ms_count += cs_stats.ms_count;
            agg.ms_scan += cs_stats.ms_scan;
            agg.ms_scatter += cs_stats.ms_scatter;
            agg.ms_canon += cs_stats.ms_canon;
        }
        DTS_CUDA(cudaStreamSynchronize(cs));
        DTS_CUDA(cudaStreamSynchronize(ds));
    } catch (...) {
        cleanup();
        pinned_free(out);
        throw;
    }
    cleanup();
    agg.results = used;
    if (stats) *stats = agg;
    if (used == 0) {
        pinned_free(out);
        out = nullptr;
    }
    *out_count = used;
    return out;
}

dts_status search_common(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                         uint32_t qid_base, cudaStream_t s, bool host, dts_result** out_results,
                         size_t* out_count, dts_search_stats* stats,
                         const dts_search_options* opts = nullptr) {
    if (out_results) *out_results = nullptr;
    if (out_count) *out_count = 0;
    dts_result* ret = nullptr;
    size_t cnt = 0;
    const uint32_t* qmap = opts ? opts->query_ids : nullptr;
    const uint32_t* qtraj = opts ? opts->query_traj : nullptr;
    const bool excl = opts && opts->exclude_same_trajectory;
    if (opts) qid_base = opts->query_id_base;
    DeviceGuard dg;
    dts_status st = guarded([&] {
        if (!index) throw Error(DTS_EINVAL, "index is NULL");
        if (!out_results || !out_count) throw Error(DTS_EINVAL, "output pointer is NULL");
        if (nq > 0 && !Q) throw Error(DTS_EINVAL, "Q is NULL with nq > 0");
        if (nq >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "nq must be < 2^32");
        if ((uint64_t)qid_base + nq > (uint64_t(1) << 32))
            throw Error(DTS_EINVAL, "query_id_base + nq exceeds 2^32");
        if (!(d >= 0.0) || !std::isfinite(d)) throw Error(DTS_EINVAL, "d must be finite and >= 0");
        prepare_device(index->device);
        SearchOut so;
        if (host) {
            DevBuf<uint32_t> dmap(qmap && nq ? nq : 0, s), dtraj(qtraj && nq ? nq : 0, s);
            if (dmap.p) {
                DTS_CUDA(cudaMemcpyAsync(dmap.p, qmap, nq * sizeof(uint32_t),
                                         cudaMemcpyHostToDevice, s));
            }
            if (dtraj.p) {
                DTS_CUDA(cudaMemcpyAsync(dtraj.p, qtraj, nq * sizeof(uint32_t),
                                         cudaMemcpyHostToDevice, s));
            }
            // large host query sets stream through the device in chunks:
            // chunk i's H2D overlaps search i-1 and its results' D2H search
            // i+1 (DTS_Q_CHUNK queries per chunk; 0 disables).  Default: from
            // 2^19 queries, chunks of max(2^18, nq / 4).  Measured on C4 (1 M
            // queries, index resident, host API): one shot 2.37 ms; chunks of
            // 131072: 2.83; 262144: 2.18; 333376: 2.25; 500064: 2.23.
            const char* ch_env = getenv("DTS_Q_CHUNK");
            const size_t chunk = ch_env ? (size_t)std::strtoull(ch_env, nullptr, 10)
                                        : (nq >= ((size_t)1 << 19)
                                               ? std::max<size_t>((size_t)1 << 18, (nq + 3) / 4)
                                               : 0);
            if (chunk > 0 && nq >= 2 * chunk) {
                try {
                    ret = search_pipelined(index, Q, nq, d, qid_base, s, chunk, dmap.p, dtraj.p,
                                           excl, stats, &cnt);
                    return;
                } catch (ResultsTooLarge&) {
                    // a chunk's results exceed the device: use the query-id
                    // streaming below (all of Q resident)
                }
            }
            DevBuf<dts_segment> dQ(nq, s);
            if (nq)
                DTS_CUDA(cudaMemcpyAsync(dQ.p, Q, nq * sizeof(dts_segment),
                                         cudaMemcpyHostToDevice, s));
            // DTS_MAX_DEVICE_RESULTS caps the results held on the device at
            // once (testing knob for the streamed path; default: memory)
            const char* cap_env = getenv("DTS_MAX_DEVICE_RESULTS");
            const unsigned long long cap = cap_env ? std::strtoull(cap_env, nullptr, 10) : ~0ull;
            try {
                search_device(index, dQ.p, nq, d, qid_base, s, &so, stats, cap ? cap : ~0ull,
                              dmap.p, dtraj.p, excl);
            } catch (ResultsTooLarge& big) {
                // stream: query-id chunks whose results fit, each searched
                // and copied out at its offset (the paper processed Q
                // incrementally when its result buffer filled)
                ret = search_streamed(index, dQ.p, nq, d, qid_base, s, big, stats, cap, dmap.p,
                                      dtraj.p, excl);
                cnt = (size_t)big.total;
                return;
            }
            if (so.count) {
                dts_result* h = nullptr;
                try {
                    h = static_cast<dts_result*>(pinned_alloc(so.count * sizeof(dts_result)));
                    copy_results_d2h(h, so.results, so.count * sizeof(dts_result), s,
                                     is_pageable_block(h));
                } catch (...) {
                    pinned_free(h);
                    cudaStreamSynchronize(s);
                    cache_free(so.results);
                    throw;
                }
                cache_free(so.results);
                ret = h;
                cnt = so.count;
            }
            DTS_CUDA(cudaStreamSynchronize(s));
        } else {
            check_aligned(Q, "Q_dev");
            search_device(index, Q, nq, d, qid_base, s, &so, stats, ~0ull, qmap, qtraj, excl);
            ret = so.results;
            cnt = so.count;
        }
    });
    if (st == DTS_OK) {
        *out_results = ret;
        *out_count = cnt;
    }
    return st;
}

// Count-only search of host or device Q: per-query counts (device buffer,
// optional copy out) and the total.
void count_common(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                  const dts_search_options* opts, cudaStream_t s, bool host_q,
                  uint32_t* counts_host, uint32_t* counts_dev_out, uint64_t* total,
                  dts_search_stats* stats) {
    const uint32_t* qtraj = opts ? opts->query_traj : nullptr;
    const bool excl = opts && opts->exclude_same_trajectory;
    DevBuf<dts_segment> dQ(host_q ? nq : 0, s);
    DevBuf<uint32_t> dtraj(host_q && qtraj && nq ? nq : 0, s), cnt(nq, s);
    const dts_segment* Qd = Q;
    if (host_q && nq) {
        DTS_CUDA(cudaMemcpyAsync(dQ.p, Q, nq * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
        Qd = dQ.p;
        if (qtraj) {
            DTS_CUDA(cudaMemcpyAsync(dtraj.p, qtraj, nq * sizeof(uint32_t),
                                     cudaMemcpyHostToDevice, s));
            qtraj = dtraj.p;
        }
    }
    SearchOut so;
    search_device(index, Qd, nq, d, 0, s, &so, stats, ~0ull, nullptr, qtraj, excl, true,
                  counts_dev_out ? counts_dev_out : cnt.p);
    if (counts_host && nq) {
        DTS_CUDA(cudaMemcpyAsync(counts_host, counts_dev_out ? counts_dev_out : cnt.p,
                                 nq * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    }
    DTS_CUDA(cudaStreamSynchronize(s));
    *total = so.count;
}

// Streamed search of host Q: a count pass plans contiguous query-id chunks of
// at most `chunk_results` results; each chunk is searched, copied to a pinned
// buffer and handed to the callback in canonical order (chunk-order
// concatenation is the canonical order).  Results never exist in full
// anywhere: the paper's incremental processing of Q.
void stream_common(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                   const dts_search_options* opts, uint64_t chunk_results,
                   dts_result_callback cb, void* user, cudaStream_t s,
                   dts_search_stats* stats) {
    const uint32_t qid_base = opts ? opts->query_id_base : 0;
    const uint32_t* qmap_h = opts ? opts->query_ids : nullptr;
    const uint32_t* qtraj_h = opts ? opts->query_traj : nullptr;
    const bool excl = opts && opts->exclude_same_trajectory;
    DevBuf<dts_segment> dQ(nq, s);
    DevBuf<uint32_t> dmap(qmap_h && nq ? nq : 0, s), dtraj(qtraj_h && nq ? nq : 0, s);
    if (nq) DTS_CUDA(cudaMemcpyAsync(dQ.p, Q, nq * sizeof(dts_segment), cudaMemcpyHostToDevice, s));
    if (dmap.p) DTS_CUDA(cudaMemcpyAsync(dmap.p, qmap_h, nq * 4, cudaMemcpyHostToDevice, s));
    if (dtraj.p) DTS_CUDA(cudaMemcpyAsync(dtraj.p, qtraj_h, nq * 4, cudaMemcpyHostToDevice, s));
    std::vector<uint32_t> counts(nq);
    DevBuf<uint32_t> dcnt(nq, s);
    dts_search_stats cst{};
    SearchOut so;
    search_device(index, dQ.p, nq, d, 0, s, &so, &cst, ~0ull, nullptr, dtraj.p, excl, true,
                  dcnt.p);
    if (nq) {
        DTS_CUDA(cudaMemcpyAsync(counts.data(), dcnt.p, nq * 4, cudaMemcpyDeviceToHost, s));
        DTS_CUDA(cudaStreamSynchronize(s));
    }
    if (chunk_results == 0) {
        size_t free_b = 0, total_b = 0;
        DTS_CUDA(cudaMemGetInfo(&free_b, &total_b));
        chunk_results = std::max<uint64_t>(1, std::min<uint64_t>(uint64_t(1) << 27,
                                                                 (uint64_t)(0.25 * free_b / 96.0)));
    }
    // pinned landing buffer: the largest chunk (a single query may exceed
    // chunk_results; it is then a chunk of its own)
    uint64_t biggest = 0;
    {
        size_t a = 0;
        while (a < nq) {
            size_t b = a;
            uint64_t acc = 0;
            while (b < nq && (b == a || acc + counts[b] <= chunk_results)) acc += counts[b++];
            biggest = std::max(biggest, acc);
            a = b;
        }
    }
    // chunks of contiguous query ids (canonical order = chunk order)
    struct Chunk {
        size_t a, b;
        uint64_t n;
    };
    std::vector<Chunk> chunks;
    {
        size_t a = 0;
        while (a < nq) {
            size_t b = a;
            uint64_t acc = 0;
            while (b < nq && (b == a || acc + counts[b] <= chunk_results)) acc += counts[b++];
            if (acc) chunks.push_back({a, b, acc});
            a = b;
        }
    }
    // two landing buffers: a worker thread searches chunk k + 1 and copies it
    // out while the caller's callback consumes chunk k
    dts_result* hbuf[2] = {nullptr, nullptr};
    dts_search_stats agg = cst;
    agg.results = 0;
    int dev = 0;
    DTS_CUDA(cudaGetDevice(&dev));
    std::mutex mu;
    std::condition_variable cv;
    size_t produced = 0, consumed = 0;
    bool stop = false;
    std::exception_ptr err;
    std::thread worker;
    try {
        for (int i = 0; i < 2 && (size_t)i < chunks.size(); ++i)
            hbuf[i] = static_cast<dts_result*>(pinned_alloc(biggest * sizeof(dts_result)));
        worker = std::thread([&] {
            try {
                DTS_CUDA(cudaSetDevice(dev));
                for (size_t k = 0; k < chunks.size(); ++k) {
                    {
                        std::unique_lock<std::mutex> lk(mu);
                        cv.wait(lk, [&] { return stop || k < consumed + 2; });
                        if (stop) return;
                    }
                    const Chunk& c = chunks[k];
                    SearchOut co;
                    search_device(index, dQ.p + c.a, c.b - c.a, d, qid_base + (uint32_t)c.a, s,
                                  &co, nullptr, ~0ull, dmap.p ? dmap.p + c.a : nullptr,
                                  dtraj.p ? dtraj.p + c.a : nullptr, excl);
                    if (co.count != c.n) {
                        cache_free(co.results);
                        throw Error(DTS_EINTERNAL, "streamed chunk count mismatch");
                    }
                    copy_results_d2h(hbuf[k & 1], co.results, c.n * sizeof(dts_result), s,
                                     is_pageable_block(hbuf[k & 1]));
                    cache_free(co.results);
                    std::lock_guard<std::mutex> lk(mu);
                    produced = k + 1;
                    cv.notify_all();
                }
            } catch (...) {
                std::lock_guard<std::mutex> lk(mu);
                err = std::current_exception();
                stop = true;
                cv.notify_all();
            }
        });
        for (size_t k = 0; k < chunks.size(); ++k) {
            {
                std::unique_lock<std::mutex> lk(mu);
                cv.wait(lk, [&] { return stop || produced > k; });
                if (produced <= k) break;                // the worker failed
            }
            agg.results += chunks[k].n;
            const bool more = cb(hbuf[k & 1], (size_t)chunks[k].n, user) == 0;
            std::lock_guard<std::mutex> lk(mu);
            consumed = k + 1;
            if (!more) stop = true;                      // the caller stops early
            cv.notify_all();
            if (!more) break;
        }
        {
            std::lock_guard<std::mutex> lk(mu);
            stop = true;
            cv.notify_all();
        }
        worker.join();
    } catch (...) {
        {
            std::lock_guard<std::mutex> lk(mu);
            stop = true;
            cv.notify_all();
        }
        if (worker.joinable()) worker.join();
        pinned_free(hbuf[0]);
        pinned_free(hbuf[1]);
        throw;
    }
    pinned_free(hbuf[0]);
    pinned_free(hbuf[1]);
    if (err) std::rethrow_exception(err);
    if (stats) *stats = agg;
}

}  // namespace
}  // namespace dts

using namespace dts;

extern "C" {

dts_status dts_build_index(const dts_segment* D, size_t n, const dts_index_params* params,
                           dts_index** out_index) {
    return build_common(D, n, params, true, cudaStreamPerThread, out_index);
}

dts_status dts_build_index_device(const dts_segment* D_dev, size_t n,
                                  const dts_index_params* params, void* cuda_stream,
                                  dts_index** out_index) {
    return build_common(D_dev, n, params, false, static_cast<cudaStream_t>(cuda_stream),
                        out_index);
}

dts_status dts_search(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                      uint32_t query_id_base, void* cuda_stream, dts_result** out_results,
                      size_t* out_count) {
    return search_common(index, Q, nq, d, query_id_base, static_cast<cudaStream_t>(cuda_stream),
                         true, out_results, out_count, nullptr);
}

dts_status dts_search_ex(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                         const dts_search_options* opts, void* cuda_stream,
                         dts_result** out_results, size_t* out_count, dts_search_stats* stats) {
    return search_common(index, Q, nq, d, 0, static_cast<cudaStream_t>(cuda_stream), true,
                         out_results, out_count, stats, opts);
}

dts_status dts_search_device_ex(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                                double d, const dts_search_options* opts, void* cuda_stream,
                                dts_result** out_results_dev, size_t* out_count,
                                dts_search_stats* stats) {
    return search_common(index, Q_dev, nq, d, 0, static_cast<cudaStream_t>(cuda_stream), false,
                         out_results_dev, out_count, stats, opts);
}

dts_status dts_merge_trajectories_device(const dts_result* results_dev, size_t n,
                                         const uint32_t* query_traj, size_t n_query_ids,
                                         const uint32_t* entry_traj, size_t n_entry_ids,
                                         void* cuda_stream, dts_traj_result** out_dev,
                                         size_t* out_count) {
    if (out_dev) *out_dev = nullptr;
    if (out_count) *out_count = 0;
    dts_traj_result* o = nullptr;
    size_t c = 0;
    DeviceGuard dg;
    dts_status st = guarded([&] {
        if (!out_dev || !out_count) throw Error(DTS_EINVAL, "output pointer is NULL");
        if (n > 0 && (!results_dev || !query_traj || !entry_traj))
            throw Error(DTS_EINVAL, "NULL input with n > 0");
        merge_trajectories_device(results_dev, n, query_traj, n_query_ids, entry_traj,
                                  n_entry_ids, static_cast<cudaStream_t>(cuda_stream), &o, &c);
    });
    if (st == DTS_OK) {
        *out_dev = o;
        *out_count = c;
    }
    return st;
}

dts_status dts_search_count(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                            const dts_search_options* opts, void* cuda_stream,
                            uint32_t* counts, uint64_t* total, dts_search_stats* stats) {
    if (total) *total = 0;
    DeviceGuard dg;
    return guarded([&] {
        if (!index) throw Error(DTS_EINVAL, "index is NULL");
        if (!total) throw Error(DTS_EINVAL, "total is NULL");
        if (nq > 0 && !Q) throw Error(DTS_EINVAL, "Q is NULL with nq > 0");
        if (nq >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "nq must be < 2^32");
        if (!(d >= 0.0) || !std::isfinite(d)) throw Error(DTS_EINVAL, "d must be finite and >= 0");
        prepare_device(index->device);
        count_common(index, Q, nq, d, opts, static_cast<cudaStream_t>(cuda_stream), true, counts,
                     nullptr, total, stats);
    });
}

dts_status dts_search_count_device(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                                   double d, const dts_search_options* opts, void* cuda_stream,
                                   uint32_t* counts_dev, uint64_t* total,
                                   dts_search_stats* stats) {
    if (total) *total = 0;
    DeviceGuard dg;
    return guarded([&] {
        if (!index) throw Error(DTS_EINVAL, "index is NULL");
        if (!total) throw Error(DTS_EINVAL, "total is NULL");
        if (nq > 0 && !Q_dev) throw Error(DTS_EINVAL, "Q_dev is NULL with nq > 0");
        if (nq >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "nq must be < 2^32");
        if (!(d >= 0.0) || !std::isfinite(d)) throw Error(DTS_EINVAL, "d must be finite and >= 0");
        prepare_device(index->device);
        if (nq) check_aligned(Q_dev, "Q_dev");
        count_common(index, Q_dev, nq, d, opts, static_cast<cudaStream_t>(cuda_stream), false,
                     nullptr, counts_dev, total, stats);
    });
}

dts_status dts_search_stream(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                             const dts_search_options* opts, uint64_t chunk_results,
                             dts_result_callback callback, void* user, void* cuda_stream,
                             dts_search_stats* stats) {
    DeviceGuard dg;
    return guarded([&] {
        if (!index) throw Error(DTS_EINVAL, "index is NULL");
        if (!callback) throw Error(DTS_EINVAL, "callback is NULL");
        if (nq > 0 && !Q) throw Error(DTS_EINVAL, "Q is NULL with nq > 0");
        if (nq >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "nq must be < 2^32");
        const uint32_t base = opts ? opts->query_id_base : 0;
        if ((uint64_t)base + nq > (uint64_t(1) << 32))
            throw Error(DTS_EINVAL, "query_id_base + nq exceeds 2^32");
        if (!(d >= 0.0) || !std::isfinite(d)) throw Error(DTS_EINVAL, "d must be finite and >= 0");
        prepare_device(index->device);
        stream_common(index, Q, nq, d, opts, chunk_results, callback, user,
                      static_cast<cudaStream_t>(cuda_stream), stats);
    });
}

dts_status dts_query_costs_sampled_device(const dts_index* index, const dts_segment* Q_dev,
                                          size_t nq, double d, uint32_t block, uint32_t stride,
                                          void* cuda_stream, uint64_t* costs_dev) {
    DeviceGuard dg;
    return guarded([&] {
        if (!index) throw Error(DTS_EINVAL, "index is NULL");
        if (nq > 0 && (!Q_dev || !costs_dev)) throw Error(DTS_EINVAL, "NULL pointer with nq > 0");
        if (nq >= (size_t(1) << 32)) throw Error(DTS_EINVAL, "nq must be < 2^32");
        if (block == 0) throw Error(DTS_EINVAL, "block must be >= 1");
        if (stride == 0) throw Error(DTS_EINVAL, "stride must be >= 1");
        if (!(d >= 0.0) || !std::isfinite(d)) throw Error(DTS_EINVAL, "d must be finite and >= 0");
        prepare_device(index->device);
        if (nq) check_aligned(Q_dev, "Q_dev");
        const cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
        query_costs_device(index, Q_dev, nq, d, block,
                           reinterpret_cast<unsigned long long*>(costs_dev), s, stride);
        DTS_CUDA(cudaStreamSynchronize(s));
    });
}

dts_status dts_query_costs_device(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                                  double d, uint32_t block, void* cuda_stream,
                                  uint64_t* costs_dev) {
    return dts_query_costs_sampled_device(index, Q_dev, nq, d, block, 1, cuda_stream, costs_dev);
}

dts_status dts_canonicalize_device(dts_result* results_dev, size_t n, void* cuda_stream) {
    return guarded([&] {
        if (n > 0 && !results_dev) throw Error(DTS_EINVAL, "results_dev is NULL with n > 0");
        canonicalize_device(results_dev, n, static_cast<cudaStream_t>(cuda_stream));
    });
}

dts_status dts_search_device(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                             double d, uint32_t query_id_base, void* cuda_stream,
                             dts_result** out_results_dev, size_t* out_count,
                             dts_search_stats* stats) {
    return search_common(index, Q_dev, nq, d, query_id_base,
                         static_cast<cudaStream_t>(cuda_stream), false, out_results_dev,
                         out_count, stats);
}

dts_status dts_search_read_times(dts_search_stats* stats) {
    return guarded([&] {
        if (!stats) throw Error(DTS_EINVAL, "stats is NULL");
        search_read_times(stats);
    });
}

void dts_free_results(dts_result* results) { pinned_free(results); }

void dts_free_results_device(void* results) {
    if (!results) return;
    // the block may still be read by work the caller enqueued on any stream
    // of its device: wait for that device (not the caller's current one)
    // before it is handed out again
    const int dev = cache_device(results);
    if (dev < 0) return;                      // not a library block
    DeviceGuard dg;
    cudaSetDevice(dev);
    cudaDeviceSynchronize();
    cache_free(results);
}

void dts_free_index(dts_index* index) {
    if (!index) return;
    free_index_memory(index);
    delete index;
}

dts_status dts_index_get_info(const dts_index* idx, dts_index_info* info) {
    return guarded([&] {
        if (!idx || !info) throw Error(DTS_EINVAL, "NULL argument");
        DeviceGuard dg;
        cudaSetDevice(idx->device);
        index_times(const_cast<dts_index*>(idx));
        dts_index_info r{};
        r.n = idx->n;
        r.shards = idx->ooc ? (uint32_t)idx->ooc->shards.size() : 0u;
        r.outlier_rows = idx->n_outliers;
        r.outlier_copies = idx->n_copies;
        r.cells = idx->n_cells;
        r.bins = (uint32_t)idx->gp.m;
        for (int a = 0; a < 3; ++a) {
            r.grid[a] = (uint32_t)idx->gp.nc[a];
            r.cell_width[a] = idx->gp.w[a];
            r.max_extent[a] = idx->max_ext[a];
        }
        r.bin_width = idx->gp.b;
        r.max_duration = idx->gp.maxdur;
        r.ms_build = idx->ms_build;
        for (int i = 0; i < 5; ++i) r.ms_phase[i] = idx->ms_phase[i];
        r.build_flags = idx->fused_keys ? 1u : 0u;
        r.hash_kind = 1u;
        r.hash_items = idx->hash_items;
        r.hash_bytes = idx->ht.slots ? (uint64_t)idx->ht.nslots() * sizeof(dts::BlockSlot) : 0;
        r.method = idx->method;
        for (int a = 0; a < 3; ++a) {
            r.subbins[a] = idx->method == DTS_METHOD_SUBBIN ? (uint32_t)idx->sb.v[a] : 0u;
            r.subbin_ids[a] = idx->sb_len[a];
        }
        *info = r;
    });
}

const char* dts_last_error(void) { return g_err.c_str(); }

const char* dts_version(void) { return "dts 0.1 (sm_100a)"; }

uint64_t dts_kernel_launches(void) { return g_launches.load(); }

}  // extern "C"
