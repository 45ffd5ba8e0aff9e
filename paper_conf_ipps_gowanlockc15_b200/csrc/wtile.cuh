// wtile.cuh -- pass 1 (fused candidate streaming + fp64 refinement, count +
// staging) and pass 2 (emission) of the search, on warp-private query tiles.
// Included by search.cu inside its anonymous namespace (uses its helpers).
//
// A warp owns a tile of WQ consecutive sorted queries and works on it alone
// (no CTA barrier): warps fetch tiles dynamically, so a warp whose queries
// sit in a dense region does not hold up others.  Per tile:
//   0. lanes 0..WQ-1 load one query each: velocity form, stencil, row-probe
//      count; a shuffle scan gives the tile's probe offsets;
//   1. rounds of 32 row probes (one per lane) -> runs; a shuffle scan flattens
//      them; lanes stream the candidates two at a time and refine them;
//      hits go to the warp's shared-memory stage (query, entry id, interval);
//   2. per-query counts are written; each staged hit's rank inside its query
//      is counted against the other staged hits (ordering by entry id), and
//      the tile's hits are written to the global stage in canonical order.
// A tile whose hits exceed WH (or the global stage) is marked for the
// count-then-scatter fallback of pass 2.

constexpr int WQ = 16;                  // queries per warp tile (32: 1.42 ms on C4, 16: 0.82)
constexpr int WH = 128;                 // staged hits per warp tile
constexpr int WT = 128;                 // threads per CTA (4 independent warps)
constexpr int WW = WT / 32;

// Query record as read by the refinement: (t0,t1) (x0,vx) (y0,vy) (z0,vz)
// in four 16-byte words (four LDS.128 per candidate instead of eight
// LDS.64), padded to 80 bytes so that queries 2 apart do not share banks.
constexpr int QREC = 5;

// A query's stencil as read by a probe lane: 64 bytes, four LDS.128.
struct __align__(16) QStencil {
    int32_t lb, hb;
    uint32_t mode, rind;
    int32_t clo[3];
    uint32_t rstart;                   // single-run queries (temporal / subbin)
    int32_t cn[3];
    uint32_t rcnt;
};

struct WarpSmem {
    double2 qrec[WQ][QREC];
    double qt0[WQ], qt1[WQ];
    QStencil qs[WQ];
    uint32_t qid[WQ], qcount[WQ], qoff[WQ];
    uint32_t qtraj[WQ];                        // trajectory ids (exclude_same_trajectory)
    unsigned long long lkoff[WQ + 1];
    unsigned long long hkey[WH];        // (query << 42) | (position, then entry id << 10) | slot
    double h0[WH], h1[WH];
    uint32_t nhit, over;
};

struct TileArgs {
    const double4* Q;
    const uint32_t* order;             // sorted position -> query id
    uint32_t nq;
    double d;
    GridParams g;
    SegSoA soa;
    HashTable ht;
    const double* bin_t0min;
    const double* bin_t1max;
    const uint32_t* bin_start;
    uint32_t* counts;                  // per query id
    dts_result* stage;                 // staged hits (tile-contiguous, canonical inside)
    unsigned long long stage_cap;
    unsigned long long* tile_base;     // per warp tile: first staged slot, NONE-1 empty, NONE redo
    uint32_t* over_tiles;              // tiles to recompute in pass 2
    uint32_t qid_base;
    const uint32_t* qmap;              // optional reported query ids (else qid + qid_base)
    const uint32_t* etraj;             // trajectory id per sorted entry position
    const uint32_t* qtraj;             // trajectory id per query row
    uint32_t excl;                     // exclude_same_trajectory
    Counters* ctr;
    uint32_t method;
    SubbinIndex sb;
};

__device__ __forceinline__ QState smem_query(const WarpSmem& S, int qi) {
    QState q;
    const double2 a = S.qrec[qi][0], b = S.qrec[qi][1], c = S.qrec[qi][2], e = S.qrec[qi][3];
    q.t0 = a.x; q.t1 = a.y;
    q.x0 = b.x; q.vx = b.y;
    q.y0 = c.x; q.vy = c.y;
    q.z0 = e.x; q.vz = e.y;
    return q;
}

// The hit is staged with its sorted position p; the entry ids of all the
// tile's hits are looked up together before ranking (one round trip per tile
// instead of a dependent load per hit).
__device__ __forceinline__ void stage_hit(WarpSmem& S, int qi, uint32_t p, double r0, double r1) {
    atomicAdd(&S.qcount[qi], 1u);
    const uint32_t pos = atomicAdd(&S.nhit, 1u);
    if (pos < (uint32_t)WH) {
        S.hkey[pos] = ((unsigned long long)qi << 42) | ((unsigned long long)p << 10) | pos;
        S.h0[pos] = r0;
        S.h1[pos] = r1;
    } else {
        S.over = 1u;
    }
}


// ---- TMA bulk staging of candidate records (sm_90+: cp.async.bulk)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
                 : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
// global -> shared bulk copy of `bytes` (multiple of 16, both 16-B aligned),
// completion counted on the mbarrier
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes,
                                         unsigned long long* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Per-warp double buffer of CH candidate records (64 B each) filled by the
// TMA engine: the candidate stream no longer goes through the LSU/L1
// (whose wavefronts run at ~70% of peak in the LDG version).
template <int CH>
struct WarpStage {
    double4 rec[2][CH][2];
    unsigned long long bar[2];
};

// SB: the subbin method (candidates through the X/Y/Z arrays); the grid and
// temporal methods compile without that indirection.  GROUP: one-run
// queries (temporal / subbin methods) streamed per group of identical runs
// (step 1a); the grid method compiles without it (its rare one-run
// fallback queries go through the probe rounds).
template <int MINB, bool TMA = false, int CH = 32, bool SB = false, bool GROUP = false>
__global__ void __launch_bounds__(WT, MINB) k_wtile_count(const TileArgs a) {
    __shared__ WarpSmem SW[WW];
    __shared__ __align__(128) WarpStage<TMA ? CH : 1> STG[TMA ? WW : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    WarpSmem& S = SW[warp];
    const GridParams& g = a.g;
    const double d = a.d, d2 = d * d;
    const uint32_t ntiles = (a.nq + WQ - 1) / WQ;
    unsigned long long n_cand = 0;
    uint32_t n_probe = 0;
    uint32_t phase[2] = {0u, 0u};
    if (TMA) {
        if (lane == 0) {
            mbar_init(&STG[warp].bar[0], 1);
            mbar_init(&STG[warp].bar[1], 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncwarp();
    }

    while (true) {
        uint32_t wt = 0;
        if (lane == 0) wt = atomicAdd(&a.ctr->work, 1u);
        wt = __shfl_sync(0xffffffffu, wt, 0);
        if (wt >= ntiles) break;

        // ---- 0: queries, stencils, probe offsets
        unsigned long long nlook = 0;
        bool single = false;                 // one-run query (temporal / subbin / fallback)
        uint32_t rs = 0, rc = 0, ri = 0;
        const uint32_t sp = wt * WQ + lane;
        if (lane < WQ) {
            QState q{};
            double qlo[3] = {0, 0, 0}, qhi[3] = {0, 0, 0};
            bool live = false;
            uint32_t qid = 0;
            if (sp < a.nq) {
                qid = a.order[sp];
                live = load_query(a.Q, qid, q, qlo, qhi);
            }
            const Stencil st = make_stencil(g, q, qlo, qhi, d, live, a.bin_start, a.bin_t0min,
                                            a.bin_t1max, a.method, a.sb);
            S.qt0[lane] = q.t0; S.qt1[lane] = q.t1;
            S.qrec[lane][0] = make_double2(q.t0, q.t1);
            S.qrec[lane][1] = make_double2(q.x0, q.vx);
            S.qrec[lane][2] = make_double2(q.y0, q.vy);
            S.qrec[lane][3] = make_double2(q.z0, q.vz);
            QStencil qs;
            qs.lb = st.lb; qs.hb = st.hb;
            qs.mode = st.mode; qs.rind = st.rind;
#pragma unroll
            for (int ax = 0; ax < 3; ++ax) { qs.clo[ax] = st.clo[ax]; qs.cn[ax] = st.cn[ax]; }
            qs.rstart = st.rstart; qs.rcnt = st.rcnt;
            S.qs[lane] = qs;
            S.qid[lane] = qid;
            S.qtraj[lane] = (a.excl && sp < a.nq) ? __ldg(a.qtraj + qid) : 0u;
            S.qcount[lane] = 0;
            nlook = st.nlook;
            if (GROUP && st.mode == MODE_TEMPORAL && st.rcnt > 0) {   // streamed in 1a
                single = true;
                nlook = 0;
                rs = st.rstart;
                rc = st.rcnt;
                ri = st.rind;
            }
        }
        if (lane == 0) { S.nhit = 0; S.over = 0; S.lkoff[0] = 0; }
        {
            unsigned long long inc = nlook;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long u = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += u;
            }
            if (lane < WQ) S.lkoff[lane + 1] = inc;
        }
        __syncwarp();
        const unsigned long long Ltot = S.lkoff[WQ];

        // ---- 1a: one-run queries grouped by identical run (sorted neighbours
        //      usually share their bins, or their subbin chunk): each
        //      candidate of a run is loaded once and refined against every
        //      query of the group, instead of once per query
        for (uint32_t smask = GROUP ? __ballot_sync(0xffffffffu, single) : 0u; smask;) {
            const int ld = __ffs(smask) - 1;
            const uint32_t lrs = __shfl_sync(0xffffffffu, rs, ld);
            const uint32_t lrc = __shfl_sync(0xffffffffu, rc, ld);
            const uint32_t lri = __shfl_sync(0xffffffffu, ri, ld);
            const uint32_t members =
                __ballot_sync(0xffffffffu, single && rs == lrs && rc == lrc && ri == lri);
            smask &= ~members;
            n_cand += (unsigned long long)__popc(members) * lrc;
            for (uint32_t base = 0; base < lrc; base += 32) {
                const uint32_t t = base + lane;
                if (t >= lrc) continue;
                const uint32_t slot = lrs + t;
                uint32_t p = slot;
                double2 st, sx, sy, sz;
                if (SB && lri) {
                    sb_load(a.sb, lri, slot, st, sx, sy, sz);
                    p = ~0u;                             // id looked up on a hit only
                    if (a.excl) p = __ldg(sb_ids(a.sb, lri) + slot);
                } else {
                    a.soa.load4(p, st, sx, sy, sz);
                }
                const uint32_t et = a.excl ? __ldg(a.etraj + p) : 0u;
                for (uint32_t mm = members; mm; mm &= mm - 1) {
                    const int qi = __ffs(mm) - 1;
                    double h0, h1;
                    if (a.excl && et == S.qtraj[qi]) continue;
                    if (refine(smem_query(S, qi), st, sx, sy, sz, d2, h0, h1)) {
                        if (p == ~0u) p = __ldg(sb_ids(a.sb, lri) + slot);
                        stage_hit(S, qi, p, h0, h1);
                    }
                }
            }
        }

        // ---- 1: rounds of 32 row probes, flattened, candidates two per lane
        for (unsigned long long r0 = 0; r0 < Ltot; r0 += 32) {
            const unsigned long long l = r0 + lane;
            uint32_t start = 0, cnt = 0, ind = 0;
            int qi = 0;
            if (l < Ltot) {
#pragma unroll
                for (int step = WQ / 2; step; step >>= 1)
                    if (S.lkoff[qi + step] <= l) qi += step;
                const uint32_t loc = (uint32_t)(l - S.lkoff[qi]);
                const QStencil qs = S.qs[qi];
                resolve(g, a.ht, a.bin_t0min, a.bin_t1max, a.bin_start, qs.mode, qs.lb,
                        qs.hb, qs.clo, qs.cn, S.qt0[qi], S.qt1[qi], loc, qs.rstart, qs.rcnt,
                        start, cnt, n_probe);
                ind = qs.rind;
            }
            unsigned long long incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long u = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += u;
            }
            const unsigned long long total = __shfl_sync(0xffffffffu, incl, 31);
            const unsigned long long excl = incl - cnt;
            n_cand += total;
            if (TMA) {
                // chunks of CH candidates: chunk c+1's runs are copied into
                // the other buffer while chunk c is refined.  Lane j copies
                // the piece of its run j that falls in the chunk.
                WarpStage<TMA ? CH : 1>& W = STG[warp];
                const unsigned long long nch = (total + CH - 1) / CH;
                auto issue = [&](unsigned long long c) {
                    const int bsel = (int)(c & 1ull);
                    const unsigned long long cb = c * CH;
                    const unsigned long long ce = min(cb + (unsigned long long)CH, total);
                    fence_proxy_async();        // our reads of this buffer precede the copy
                    if (lane == 0) mbar_expect_tx(&W.bar[bsel], (uint32_t)((ce - cb) * 64));
                    __syncwarp();
                    const unsigned long long lo = max(excl, cb), hi = min(incl, ce);
                    if (hi > lo)
                        bulk_g2s(&W.rec[bsel][lo - cb][0],
                                 a.soa.rec + 4 * ((size_t)start + (size_t)(lo - excl)),
                                 (uint32_t)((hi - lo) * 64), &W.bar[bsel]);
                };
                if (nch) issue(0);    // (an empty round issues nothing: every
                                      //  expect_tx must be matched by a wait)
                for (unsigned long long c = 0; c < nch; ++c) {
                    if (c + 1 < nch) issue(c + 1);
                    const int bsel = (int)(c & 1ull);
                    mbar_wait(&W.bar[bsel], phase[bsel]);
                    phase[bsel] ^= 1u;
                    const unsigned long long cb = c * CH;
#pragma unroll
                    for (int h = 0; h < CH / 32; ++h) {
                        const unsigned long long t1 = cb + lane + 32 * h;
                        int j1 = 0;
#pragma unroll
                        for (int step = 16; step; step >>= 1)
                            if (__shfl_sync(0xffffffffu, incl, j1 + step - 1) <= t1) j1 += step;
                        const uint32_t s1 = __shfl_sync(0xffffffffu, start, j1);
                        const unsigned long long e1 = __shfl_sync(0xffffffffu, excl, j1);
                        const int qi1 = __shfl_sync(0xffffffffu, qi, j1);
                        if (t1 < total) {
                            const uint32_t p1 = s1 + (uint32_t)(t1 - e1);
                            const double4 r0 = W.rec[bsel][lane + 32 * h][0];
                            const double4 r1 = W.rec[bsel][lane + 32 * h][1];
                            double h0, h1;
                            const bool x1 = a.excl && __ldg(a.etraj + p1) == S.qtraj[qi1];
                            if (!x1 && refine(smem_query(S, qi1), make_double2(r0.x, r0.y),
                                              make_double2(r0.z, r0.w), make_double2(r1.x, r1.y),
                                              make_double2(r1.z, r1.w), d2, h0, h1))
                                stage_hit(S, qi1, p1, h0, h1);
                        }
                    }
                    __syncwarp();
                }
            } else {
            // per run: the position delta start - excl (mod 2^32: a candidate's
            // position p = t + delta fits 32 bits even when the round's total
            // does not) and (query | method index << 8), one 32-bit shuffle
            // each; the run search shuffles 32-bit prefixes when the total fits
            const uint32_t delta = start - (uint32_t)excl;
            const uint32_t qind = (uint32_t)qi | (ind << 8);
            const bool narrow = total <= 0xffffffffull;
            const uint32_t incl32 = (uint32_t)incl;
            for (unsigned long long base = 0; base < total; base += 64) {
                const unsigned long long t1 = base + lane, t2 = t1 + 32;
                int j1 = 0, j2 = 0;
                if (narrow) {
                    const uint32_t u1 = (uint32_t)t1, u2 = (uint32_t)t2;
#pragma unroll
                    for (int step = 16; step; step >>= 1) {
                        if (__shfl_sync(0xffffffffu, incl32, j1 + step - 1) <= u1) j1 += step;
                        if (__shfl_sync(0xffffffffu, incl32, j2 + step - 1) <= u2) j2 += step;
                    }
                } else {
#pragma unroll
                    for (int step = 16; step; step >>= 1) {
                        if (__shfl_sync(0xffffffffu, incl, j1 + step - 1) <= t1) j1 += step;
                        if (__shfl_sync(0xffffffffu, incl, j2 + step - 1) <= t2) j2 += step;
                    }
                }
                const uint32_t dl1 = __shfl_sync(0xffffffffu, delta, j1);
                const uint32_t dl2 = __shfl_sync(0xffffffffu, delta, j2);
                const uint32_t qx1 = __shfl_sync(0xffffffffu, qind, j1);
                const uint32_t qx2 = __shfl_sync(0xffffffffu, qind, j2);
                const int qi1 = (int)(qx1 & 0xffu), qi2 = (int)(qx2 & 0xffu);
                const uint32_t i1 = SB ? qx1 >> 8 : 0u, i2 = SB ? qx2 >> 8 : 0u;
                const bool v1 = t1 < total, v2 = t2 < total;
                if (v1) {
                    uint32_t p1 = (uint32_t)t1 + dl1;
                    uint32_t p2 = v2 ? (uint32_t)t2 + dl2 : p1;
                    const uint32_t i2v = v2 ? i2 : i1;
                    const uint32_t sl1 = p1, sl2 = p2;      // subbin slots (when i != 0)
                    if (i1) p1 = __ldg(sb_ids(a.sb, i1) + sl1);   // id -> sorted position
                    if (v2 && i2) p2 = __ldg(sb_ids(a.sb, i2) + sl2);
                    else if (!v2) p2 = p1;
                    double2 st1, sx1, sy1, sz1, st2, sx2, sy2, sz2;
                    if (i1) sb_load(a.sb, i1, sl1, st1, sx1, sy1, sz1);   // contiguous copy
                    else a.soa.load4(p1, st1, sx1, sy1, sz1);
                    if (i2v) sb_load(a.sb, i2v, v2 ? sl2 : sl1, st2, sx2, sy2, sz2);
                    else a.soa.load4(p2, st2, sx2, sy2, sz2);
                    double h0, h1;
                    const bool x1 = a.excl && __ldg(a.etraj + p1) == S.qtraj[qi1];
                    const bool x2 = a.excl && __ldg(a.etraj + p2) == S.qtraj[qi2];
                    if (!x1 && refine(smem_query(S, qi1), st1, sx1, sy1, sz1, d2, h0, h1))
                        stage_hit(S, qi1, p1, h0, h1);
                    if (v2 && !x2 &&
                        refine(smem_query(S, qi2), st2, sx2, sy2, sz2, d2, h0, h1))
                        stage_hit(S, qi2, p2, h0, h1);
                }
            }
            }
        }
        __syncwarp();

        // ---- 2: counts, canonical staging
        const uint32_t nh = S.nhit;
        const uint32_t cnt = lane < WQ ? S.qcount[lane] : 0u;
        if (lane < WQ && sp < a.nq) {
            a.counts[S.qid[lane]] = cnt;
            if (cnt) atomicMax(&a.ctr->max_count, cnt);
        }
        bool over = S.over != 0u;
        if (!over && nh > 0) {
            uint32_t inc = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += u;
            }
            if (lane < WQ) S.qoff[lane] = inc - cnt;
            for (uint32_t i = lane; i < nh; i += 32) {      // sorted position -> entry id
                const unsigned long long k = S.hkey[i];
                const uint32_t e = __ldg(a.soa.eid + (uint32_t)(k >> 10));
                S.hkey[i] = (k & ~(0xffffffffull << 10)) | ((unsigned long long)e << 10);
            }
            unsigned long long b = 0;
            if (lane == 0) b = atomicAdd(&a.ctr->staged, (unsigned long long)nh);
            b = __shfl_sync(0xffffffffu, b, 0);
            over = b + nh > a.stage_cap;
            __syncwarp();
            if (!over) {
                for (uint32_t i = lane; i < nh; i += 32) {
                    const unsigned long long k = S.hkey[i];
                    const uint32_t q = (uint32_t)(k >> 42), e = (uint32_t)(k >> 10);
                    // rank inside the query: hits with a smaller entry id,
                    // ties (equal caller ids) broken by stage slot, so every
                    // slot of the tile's range is written exactly once
                    uint32_t rank = 0;
                    for (uint32_t j = 0; j < nh; ++j) {
                        const unsigned long long kj = S.hkey[j];
                        const uint32_t ej = (uint32_t)(kj >> 10);
                        rank += ((uint32_t)(kj >> 42) == q && (ej < e || (ej == e && j < i))) ? 1u : 0u;
                    }
                    const uint32_t slot = (uint32_t)(k & 1023ull);
                    dts_result r;
                    r.query_id = a.qmap ? __ldg(a.qmap + S.qid[q]) : S.qid[q] + a.qid_base;
                    r.entry_id = e;
                    r.t_start = S.h0[slot];
                    r.t_end = S.h1[slot];
                    a.stage[b + S.qoff[q] + rank] = r;
                }
                if (lane == 0) a.tile_base[wt] = b;
            }
        } else if (!over && lane == 0) {
            a.tile_base[wt] = NONE - 1;          // no hits: nothing to emit
        }
        if (over) {
            if (lane == 0) {
                a.tile_base[wt] = NONE;
                const uint32_t slot = atomicAdd(&a.ctr->n_over, 1u);
                a.over_tiles[slot] = wt;
            }
        }
        __syncwarp();
    }

    // ---- statistics
    unsigned long long pr = n_probe;
#pragma unroll
    for (int o = 16; o; o >>= 1) pr += __shfl_xor_sync(0xffffffffu, pr, o);
    if (lane == 0 && pr) atomicAdd(&a.ctr->lookups, pr);
    if (lane == 0 && n_cand) atomicAdd(&a.ctr->candidates, n_cand);
}

// ------------------------------------------------------ pass 2: emission
// One warp per warp tile: the tile's staged hits are contiguous and grouped
// by query in canonical order; copy each query's group to its exact offset.
__global__ void __launch_bounds__(WT) k_wtile_emit(const uint32_t* __restrict__ order, uint32_t nq,
                                                  const uint32_t* __restrict__ counts,
                                                  const unsigned long long* __restrict__ offsets,
                                                  const unsigned long long* __restrict__ tile_base,
                                                  const dts_result* __restrict__ stage,
                                                  dts_result* __restrict__ out) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t ntiles = (nq + WQ - 1) / WQ;
    const uint32_t wt = blockIdx.x * WW + warp;
    if (wt >= ntiles) return;
    const unsigned long long tb = tile_base[wt];
    if (tb >= NONE - 1) return;                      // recomputed or empty tile
    const uint32_t sp = wt * WQ + lane;
    uint32_t cnt = 0;
    unsigned long long off = 0;
    if (lane < WQ && sp < nq) {
        const uint32_t qid = order[sp];
        cnt = counts[qid];
        off = offsets[qid];
    }
    uint32_t incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += u;
    }
    const uint32_t excl = incl - cnt;
    const uint32_t nh = __shfl_sync(0xffffffffu, incl, 31);
    for (uint32_t base = 0; base < nh; base += 32) {
        const uint32_t i = base + lane;
        int q = 0;
#pragma unroll
        for (int step = 16; step; step >>= 1)
            if (__shfl_sync(0xffffffffu, incl, q + step - 1) <= i) q += step;
        const unsigned long long o = __shfl_sync(0xffffffffu, off, q);
        const uint32_t e = __shfl_sync(0xffffffffu, excl, q);
        if (i < nh) out[o + (i - e)] = stage[tb + i];
    }
}
