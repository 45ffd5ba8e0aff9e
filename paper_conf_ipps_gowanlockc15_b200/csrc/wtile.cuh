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
//      hits go to the warp's shared-memory stage (query, position, interval);
//   2. per-query counts are written; each staged hit's rank inside its query
//      is counted against the other staged hits (ordering by entry id), and
//      the tile's hits are written to the global stage in canonical order.
// Output-heavy tiles: whenever the shared stage could overflow in the next
// step (more than WH - 64 hits), the warp flushes it to a global spill buffer
// (one atomic per flush; hits as final records with the local query id) and
// goes on; after the scan the spilled records are placed at their query's
// offsets and each such query's segment is sorted by entry id (k_spill_place,
// k_seg_sort).  No candidate is streamed twice.  Only a tile that finds the
// spill buffer full is re-run (pass 1 again over the listed tiles, spilling
// every hit into an exactly sized second buffer).

constexpr int WQ = 16;                  // queries per warp tile (32: 1.42 ms on C4, 16: 0.82)
constexpr int WH = 128;                 // staged hits per warp tile
constexpr int WT = 128;                 // threads per CTA (4 independent warps)
constexpr int WW = WT / 32;
constexpr unsigned long long SPILLED = NONE - 2;   // tile_base of a spilled tile

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
    uint2 run[32];                      // a probe round's non-empty runs, compacted:
                                        // (position delta, query | method index << 8)
    uint32_t nhit, over, spilled;
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
    unsigned long long* tile_base;     // per warp tile: first staged slot, NONE-1 empty,
                                       // SPILLED spilled, NONE re-run
    uint32_t* over_tiles;              // tiles to re-run (spill buffer full)
    uint32_t* spill_tiles;             // tiles whose hits went to the spill buffer
    uint2* spill_qe;                   // spilled hits: (LOCAL query id, entry id) ...
    double2* spill_t;                  // ... and their interval (two arrays: the
                                       // placement reads only the ids)
    unsigned long long spill_cap;
    const uint32_t* tile_list;         // re-run: the tiles to process (else 0..ntiles-1)
    uint32_t n_list;
    uint32_t spill_all;                // re-run: every hit is spilled
    uint32_t count_only;               // per-query counts only (no hit is kept)
    uint32_t qid_base;
    const uint32_t* qmap;              // optional reported query ids (else qid + qid_base)
    const uint32_t* etraj;             // trajectory id per sorted entry position
    const uint32_t* qtraj;             // trajectory id per query row
    uint32_t excl;                     // exclude_same_trajectory
    Counters* ctr;
    uint32_t method;
    SubbinIndex sb;
    OutlierIndex out;                  // long-segment copies (okeys NULL: none)
    unsigned long long* qstage;        // per query id: first staged slot (pass 2), or NULL
    uint32_t tq;                       // queries per tile (1..WQ; fewer on small query sets)
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
// instead of a dependent load per hit).  A tile that is to be re-run only
// counts.
__device__ __forceinline__ void stage_hit(WarpSmem& S, int qi, uint32_t p, double r0, double r1) {
    atomicAdd(&S.qcount[qi], 1u);
    if (S.over) return;
    const uint32_t pos = atomicAdd(&S.nhit, 1u);
    if (pos < (uint32_t)WH) {
        S.hkey[pos] = ((unsigned long long)qi << 42) | ((unsigned long long)p << 10) | pos;
        S.h0[pos] = r0;
        S.h1[pos] = r1;
    } else {
        S.over = 1u;
    }
}

// A hit on position p counts unless p holds a copy of an outlier that is not
// the query's canonical copy (internal.cuh "outliers"): the least key among
// the sub-slice boxes of the first bin the query probes whose boxes meet its
// stencil box (the whole grid for a query that scans its bins' full range).
// A pair within d is met in that bin and cell by construction, and copies
// with equal packed keys (a repeated cell, or the midpoint filing) keep the
// first position only: exactly one copy of each outlier yields the hit.
struct OutlierArgs {                  // what the canonical-copy test reads
    OutlierIndex out;
    SegSoA soa;
    const double* bin_t0min;
    const double* bin_t1max;
};

// Whether the copy at position p is the query's canonical copy of its
// outlier.  Out of line: called for hits on outlier copies only.
__device__ __noinline__ bool outlier_canonical(const OutlierArgs* __restrict__ ap,
                                               const GridParams* __restrict__ gp,
                                               const QStencil* __restrict__ qsp, double qt0,
                                               double qt1, uint32_t p) {
    const OutlierArgs& a = *ap;
    const GridParams& g = *gp;
    const unsigned long long pk = __ldg(a.out.okeys + p);
    if (p > 0 && __ldg(a.out.okeys + p - 1) == pk) return false;                // repeated copy
    const unsigned long long key = pk >> a.out.shift;
    const QStencil qs = *qsp;
    double2 st, sx, sy, sz;
    a.soa.load4(p, st, sx, sy, sz);
    ORec o;
    o.t0 = st.x; o.t1 = st.y;
    o.x[0] = sx.x; o.x[1] = sy.x; o.x[2] = sz.x;
    o.v[0] = sx.y; o.v[1] = sy.y; o.v[2] = sz.y;
    const int32_t jo0 = bin_of(g, o.t0), jo1 = bin_of(g, o.t1);
    int32_t blo[3], bhi[3];
    for (int ax = 0; ax < 3; ++ax) {
        const bool grid = qs.mode == MODE_GRID;
        blo[ax] = grid ? qs.clo[ax] : 0;
        bhi[ax] = grid ? qs.clo[ax] + qs.cn[ax] - 1 : g.nc[ax] - 1;
    }
    for (int32_t j = max(qs.lb, jo0); j <= min(qs.hb, jo1); ++j) {
        // interior bins a row probe skips (extent not overlapping the query)
        if (qs.mode == MODE_GRID && j != qs.lb && j != qs.hb &&
            !(__ldg(&a.bin_t0min[j]) < qt1 && __ldg(&a.bin_t1max[j]) > qt0))
            continue;
        unsigned long long best = ~0ull;
        outlier_boxes(g, o, j, jo0, jo1, [&](const int32_t lo[3], const int32_t hi[3]) {
            const int32_t cx = max(lo[0], blo[0]), cy = max(lo[1], blo[1]), cz = max(lo[2], blo[2]);
            if (cx <= min(hi[0], bhi[0]) && cy <= min(hi[1], bhi[1]) && cz <= min(hi[2], bhi[2])) {
                const unsigned long long k = make_key(g, j, cx, cy, cz);
                best = k < best ? k : best;
            }
        });
        if (best != ~0ull) return best == key;
    }
    return false;
}

__device__ __forceinline__ bool is_copy(const OutlierIndex& out, uint32_t p) {
    return (__ldg(out.obits + (p >> 5)) >> (p & 31u)) & 1u;
}

// Warp-uniform, only for indexes with outliers: every staged hit's entry id
// and copy flag are loaded together (one round trip, as the plain path's id
// lookup); hits on copies that are not the query's canonical copy are
// dropped, the stage compacted, the query counts corrected, and the kept
// hits' positions replaced by their entry ids (hkey then holds entry ids).
__device__ __forceinline__ void filter_resolve_ids(WarpSmem& S, const OutlierArgs* oa,
                                                   const GridParams* og, int lane) {
    __syncwarp();
    const uint32_t nh = min(S.nhit, (uint32_t)WH);
    uint32_t kept = 0;
    for (uint32_t b0 = 0; b0 < nh; b0 += 32) {
        const uint32_t i = b0 + lane;
        bool keep = false;
        unsigned long long k = 0;
        double r0 = 0.0, r1 = 0.0;
        uint32_t e = 0;
        if (i < nh) {
            k = S.hkey[i];
            r0 = S.h0[i];
            r1 = S.h1[i];
            const uint32_t p = (uint32_t)(k >> 10);
            e = __ldg(oa->soa.eid + p);
            keep = true;
            if (is_copy(oa->out, p)) {
                const int qi = (int)(k >> 42);
                keep = outlier_canonical(oa, og, &S.qs[qi], S.qt0[qi], S.qt1[qi], p);
                if (!keep) atomicSub(&S.qcount[qi], 1u);
            }
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, keep);
        __syncwarp();
        if (keep) {                               // compact in place (targets <= sources)
            const uint32_t dst = kept + __popc(bal & ((1u << lane) - 1u));
            S.hkey[dst] = (k & (0xFull << 42)) | ((unsigned long long)e << 10) | dst;
            S.h0[dst] = r0;
            S.h1[dst] = r1;
        }
        kept += __popc(bal);
        __syncwarp();
    }
    if (lane == 0) S.nhit = kept;
    __syncwarp();
}

// Warp-uniform: the shared stage's hits -> the global spill buffer as
// records (local query id, entry id, interval); one atomic per flush.  A
// flush that finds the buffer full marks the tile for a re-run and records
// the first invalid slot (records from there on are not placed).  OUT: the
// record carries the hit's sorted position instead of the entry id, and the
// tile's counts include hits on non-canonical copies; k_spill_filter
// resolves and filters the records before the scan (no out-of-line call in
// the streaming loop: measured on C4 + 0.01 % long segments, the filter
// called from here cost 0.075 ms of pass 1 in spilled registers).
template <bool OUT>
__device__ __forceinline__ void flush_spill(WarpSmem& S, const TileArgs& a, int lane) {
    __syncwarp();
    const uint32_t nh = min(S.nhit, (uint32_t)WH);
    if (nh == 0 || S.over) return;
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(&a.ctr->spilled, (unsigned long long)nh);
    b = __shfl_sync(0xffffffffu, b, 0);
    if (b + nh > a.spill_cap) {
        if (lane == 0) {
            atomicMin(&a.ctr->spill_valid, b);
            S.over = 1u;
        }
        __syncwarp();
        return;
    }
    for (uint32_t i = lane; i < nh; i += 32) {
        const unsigned long long k = S.hkey[i];
        a.spill_qe[b + i] = make_uint2(S.qid[(uint32_t)(k >> 42)],
                                       OUT ? (uint32_t)(k >> 10) : __ldg(a.soa.eid + (uint32_t)(k >> 10)));
        a.spill_t[b + i] = make_double2(S.h0[i], S.h1[i]);
    }
    __syncwarp();
    if (lane == 0) {
        S.nhit = 0;
        S.spilled = 1u;
    }
    __syncwarp();
}

// A hit of the probe rounds: staged; in count-only mode on an index with
// outlier copies, checked against the canonical copy right away (nothing is
// staged to be filtered later).
template <bool OUT, bool CNT>
__device__ __forceinline__ void record_hit(WarpSmem& S, const TileArgs& a, int qi, uint32_t p,
                                           double r0, double r1, const OutlierArgs* oa,
                                           const GridParams* og) {
    if constexpr (OUT && CNT) {
        if (!is_copy(a.out, p) ||
            outlier_canonical(oa, og, &S.qs[qi], S.qt0[qi], S.qt1[qi], p))
            atomicAdd(&S.qcount[qi], 1u);
        return;
    }
    stage_hit(S, qi, p, r0, r1);
}

// Flush when the next step (at most `step_max` hits) could overflow the stage.
template <bool OUT>
__device__ __forceinline__ void maybe_flush(WarpSmem& S, const TileArgs& a, int lane,
                                            uint32_t step_max) {
    __syncwarp();
    if (S.nhit > (uint32_t)WH - step_max) flush_spill<OUT>(S, a, lane);
}

// One probe round's runs (lane: [start, start + cnt) of query qi, subbin
// array ind - 1 or sorted positions when 0), flattened and streamed two
// candidates per lane; hits staged (or spilled).
template <bool SB, bool EXCL, bool OUT, bool CNT>
__device__ __forceinline__ void stream_round(WarpSmem& S, const TileArgs& a, int lane,
                                             uint32_t start, uint32_t cnt, int qi, uint32_t ind,
                                             double d2, unsigned long long& n_cand,
                                             const OutlierArgs* s_oa, const GridParams* s_g) {
    unsigned long long incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long u = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += u;
    }
    const unsigned long long total = __shfl_sync(0xffffffffu, incl, 31);
    const unsigned long long excl = incl - cnt;
    n_cand += total;
    // the round's non-empty runs, compacted into shared memory:
    // (position delta start - excl mod 2^32, query | method index <<
    // 8); a candidate t lies in run r = (non-empty runs starting at
    // or before t) - 1, counted with one OR-reduction of the run
    // starts per 32 candidates -- no per-candidate search
    const bool ne = cnt > 0;
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t nemask = __ballot_sync(0xffffffffu, ne);
    if (ne) S.run[__popc(nemask & lt)] = make_uint2(start - (uint32_t)excl,
                                                    (uint32_t)qi | (ind << 8));
    __syncwarp();
    uint32_t before = 0;          // non-empty runs starting before `base`
    for (unsigned long long base = 0; base < total; base += 64) {
        // run-start offsets inside the two 32-candidate halves
        const unsigned long long o1 = excl - base, o2 = o1 - 32;
        const uint32_t m1 = __reduce_or_sync(0xffffffffu, (ne && excl >= base && o1 < 32)
                                                              ? 1u << (uint32_t)o1 : 0u);
        const uint32_t m2 = __reduce_or_sync(
            0xffffffffu, (ne && excl >= base + 32 && o2 < 32) ? 1u << (uint32_t)o2 : 0u);
        const uint32_t r1 = min(before + __popc(m1 & (lt | (1u << lane))) - 1u, 31u);
        before += __popc(m1);
        const uint32_t r2 = min(before + __popc(m2 & (lt | (1u << lane))) - 1u, 31u);
        before += __popc(m2);
        const unsigned long long t1 = base + lane, t2 = t1 + 32;
        const bool v1 = t1 < total, v2 = t2 < total;
        if (v1) {
            const uint2 ru1 = S.run[r1];
            const uint2 ru2 = v2 ? S.run[r2] : ru1;
            const int qi1 = (int)(ru1.y & 0xffu), qi2 = (int)(ru2.y & 0xffu);
            const uint32_t i1 = SB ? ru1.y >> 8 : 0u, i2 = SB ? ru2.y >> 8 : 0u;
            uint32_t p1 = (uint32_t)t1 + ru1.x;
            uint32_t p2 = v2 ? (uint32_t)t2 + ru2.x : p1;
            const uint32_t sl1 = p1, sl2 = p2;      // subbin slots (when i != 0)
            if (i1) p1 = __ldg(sb_ids(a.sb, i1) + sl1);   // id -> sorted position
            if (v2 && i2) p2 = __ldg(sb_ids(a.sb, i2) + sl2);
            else if (!v2) p2 = p1;
            double2 st1, sx1, sy1, sz1, st2, sx2, sy2, sz2;
            if (i1) sb_load(a.sb, i1, sl1, st1, sx1, sy1, sz1);   // contiguous copy
            else a.soa.load4(p1, st1, sx1, sy1, sz1);
            if (i2) sb_load(a.sb, i2, sl2, st2, sx2, sy2, sz2);
            else a.soa.load4(p2, st2, sx2, sy2, sz2);
            double h0, h1;
            const bool x1 = EXCL && __ldg(a.etraj + p1) == S.qtraj[qi1];
            const bool x2 = EXCL && __ldg(a.etraj + p2) == S.qtraj[qi2];
            if (!x1 && refine(smem_query(S, qi1), st1, sx1, sy1, sz1, d2, h0, h1))
                record_hit<OUT, CNT>(S, a, qi1, p1, h0, h1, s_oa, s_g);
            if (v2 && !x2 &&
                refine(smem_query(S, qi2), st2, sx2, sy2, sz2, d2, h0, h1))
                record_hit<OUT, CNT>(S, a, qi2, p2, h0, h1, s_oa, s_g);
        }
        maybe_flush<OUT>(S, a, lane, 64u);
    }
}

// Step 2 of a tile: counts; canonical staging, or the last spill flush.
template <bool OUT>
__device__ __forceinline__ void tile_finish(WarpSmem& S, const TileArgs& a, int lane, uint32_t wt,
                                            uint32_t sp, const OutlierArgs* s_oa,
                                            const GridParams* s_g) {
    // (OUT: a staged tile's ids are resolved, and its hits on
    //  non-canonical copies dropped, before the counts are read; a
    //  spilled tile's counts are corrected by k_spill_filter, and their
    //  maximum taken by k_spill_max after it)
    if constexpr (OUT) {
        if (!S.over && !a.count_only && !S.spilled && !a.spill_all)
            filter_resolve_ids(S, s_oa, s_g, lane);
    }
    const bool mine = lane < a.tq && sp < a.nq;
    const uint32_t cnt = mine ? S.qcount[lane] : 0u;
    if (mine) {
        a.counts[S.qid[lane]] = cnt;
        if (cnt && !(OUT && S.spilled)) atomicMax(&a.ctr->max_count, cnt);
    }
    if (a.spill_all || S.spilled) flush_spill<OUT>(S, a, lane);
    __syncwarp();
    const uint32_t nh = S.nhit;
    bool over = S.over != 0u;
    unsigned long long sbase = NONE;          // the tile's staged range, when staged
    if (a.spill_all) {
        // re-run: every hit is in the spill buffer (exactly sized)
    } else if (!over && S.spilled) {
        if (lane == 0) {
            a.tile_base[wt] = SPILLED;
            a.spill_tiles[atomicAdd(&a.ctr->n_spill, 1u)] = wt;
        }
    } else if (!over && nh > 0) {
        uint32_t inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        if (lane < WQ) S.qoff[lane] = inc - cnt;
        if (!OUT) {
            for (uint32_t i = lane; i < nh; i += 32) {  // sorted position -> entry id
                const unsigned long long k = S.hkey[i];
                const uint32_t e = __ldg(a.soa.eid + (uint32_t)(k >> 10));
                S.hkey[i] = (k & ~(0xffffffffull << 10)) | ((unsigned long long)e << 10);
            }
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
                // (a query with one staged hit -- most of them on the
                // galaxy workloads -- has rank 0)
                uint32_t rank = 0;
                if (S.qcount[q] > 1u) {
                    for (uint32_t j = 0; j < nh; ++j) {
                        const unsigned long long kj = S.hkey[j];
                        const uint32_t ej = (uint32_t)(kj >> 10);
                        rank += ((uint32_t)(kj >> 42) == q && (ej < e || (ej == e && j < i))) ? 1u : 0u;
                    }
                }
                const uint32_t slot = (uint32_t)(k & 1023ull);
                DTS_DCHECK(slot < (uint32_t)WH && rank < S.qcount[q] &&
                           b + S.qoff[q] + rank < a.stage_cap && b + S.qoff[q] + rank < b + nh);
                dts_result r;
                r.query_id = a.qmap ? __ldg(a.qmap + S.qid[q]) : S.qid[q] + a.qid_base;
                r.entry_id = e;
                r.t_start = S.h0[slot];
                r.t_end = S.h1[slot];
                a.stage[b + S.qoff[q] + rank] = r;
            }
            if (lane == 0) a.tile_base[wt] = b;
            sbase = b;
        }
    } else if (!over && lane == 0) {
        a.tile_base[wt] = NONE - 1;          // no hits: nothing to emit
    }
    if (over && !a.spill_all && !a.count_only && lane == 0) {
        a.tile_base[wt] = NONE;
        a.over_tiles[atomicAdd(&a.ctr->n_over, 1u)] = wt;
    }
    // per query id: where its staged hits start (NONE: spilled or re-run,
    // placed by the spill path), for pass 2's gather
    if (a.qstage && !a.spill_all && mine && cnt) {
        DTS_DCHECK(S.qid[lane] < a.nq && (sbase == NONE || cnt <= (uint32_t)WH));
        a.qstage[S.qid[lane]] = sbase == NONE ? NONE : sbase + S.qoff[lane];
    }
}

// SB: the subbin method (candidates through the X/Y/Z arrays); the grid and
// temporal methods compile without that indirection.  GROUP: one-run
// queries (temporal / subbin methods) streamed per group of identical runs
// (step 1a); the grid method compiles without it (its rare one-run
// fallback queries go through the probe rounds).  EXCL: exclude pairs of
// the same trajectory (compiled out of the plain search).  OUT: the index
// has long-segment copies (the canonical-copy filter of the hits); CNT:
// count-only search on such an index (the filter applied at each hit).
template <int MINB, bool SB = false, bool GROUP = false, bool EXCL = false, bool OUT = false,
          bool CNT = false>
__global__ void __launch_bounds__(WT, MINB) k_wtile_count(const TileArgs a) {
    __shared__ WarpSmem SW[WW];
    // the grid and the outlier arrays in shared memory for the (out-of-line)
    // canonical-copy filter: passing the kernel parameters' address would
    // copy all of them to the stack
    __shared__ GridParams s_g[OUT ? 1 : 1];
    __shared__ OutlierArgs s_oa[OUT ? 1 : 1];
    if (OUT) {
        if (threadIdx.x == 0) {
            s_g[0] = a.g;
            s_oa[0] = OutlierArgs{a.out, a.soa, a.bin_t0min, a.bin_t1max};
        }
        __syncthreads();
    }
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    WarpSmem& S = SW[warp];
    const GridParams& g = a.g;
    const double d = a.d, d2 = d * d;
    const uint32_t ntiles = a.tile_list ? a.n_list : (a.nq + a.tq - 1) / a.tq;
    unsigned long long n_cand = 0;
    uint32_t n_probe = 0;

    while (true) {
        uint32_t wi = 0;
        if (lane == 0) wi = atomicAdd(&a.ctr->work, 1u);
        wi = __shfl_sync(0xffffffffu, wi, 0);
        if (wi >= ntiles) break;
        const uint32_t wt = a.tile_list ? a.tile_list[wi] : wi;

        // ---- 0: queries, stencils, probe offsets
        unsigned long long nlook = 0;
        bool single = false;                 // one-run query (temporal / subbin / fallback)
        uint32_t rs = 0, rc = 0, ri = 0;
        const uint32_t sp = wt * a.tq + lane;
        if (lane < WQ) {
            QState q{};
            double qlo[3] = {0, 0, 0}, qhi[3] = {0, 0, 0};
            bool live = false;
            uint32_t qid = 0;
            if (lane < a.tq && sp < a.nq) {
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
            S.qtraj[lane] = (EXCL && lane < a.tq && sp < a.nq) ? __ldg(a.qtraj + qid) : 0u;
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
        if (lane == 0) { S.nhit = 0; S.over = a.count_only; S.spilled = 0; S.lkoff[0] = 0; }
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
        //      query of the group, instead of once per query; at most 32
        //      hits per (candidate chunk, query) step
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
                const bool valid = t < lrc;
                const uint32_t slot = lrs + (valid ? t : 0u);
                uint32_t p = slot;
                double2 st = make_double2(0, 0), sx = st, sy = st, sz = st;
                if (valid) {
                    if (SB && lri) {
                        sb_load(a.sb, lri, slot, st, sx, sy, sz);
                        p = ~0u;                             // id looked up on a hit only
                        if (EXCL) p = __ldg(sb_ids(a.sb, lri) + slot);
                    } else {
                        a.soa.load4(p, st, sx, sy, sz);
                    }
                }
                const uint32_t et = (EXCL && valid) ? __ldg(a.etraj + p) : 0u;
                for (uint32_t mm = members; mm; mm &= mm - 1) {
                    const int qi = __ffs(mm) - 1;
                    double h0, h1;
                    if (valid && !(EXCL && et == S.qtraj[qi]) &&
                        refine(smem_query(S, qi), st, sx, sy, sz, d2, h0, h1)) {
                        if (p == ~0u) p = __ldg(sb_ids(a.sb, lri) + slot);
                        stage_hit(S, qi, p, h0, h1);
                    }
                    maybe_flush<OUT>(S, a, lane, 32u);
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
            stream_round<SB, EXCL, OUT, CNT>(S, a, lane, start, cnt, qi, ind, d2, n_cand, s_oa, s_g);
        }
        __syncwarp();

        tile_finish<OUT>(S, a, lane, wt, sp, s_oa, s_g);
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
// Pass 2 as a gather: a warp per 32 consecutive query ids.  The warp's
// staged queries (at most WH hits each: a staged tile holds at most WH) are
// numbered by a shuffle scan of their counts; lane j of each 32-record step
// finds its query by a shuffle search of that scan and copies the query's
// staged record to its exact offset (queries ascend, so the writes of a
// step are contiguous unless a spilled query sits in between).  Queries of
// spilled or re-run tiles (qstage NONE) are left to the spill path; slots
// from cap on are not written (speculative launch).
__global__ void __launch_bounds__(256) k_emit_gather(uint32_t nq,
                                                    const uint32_t* __restrict__ counts,
                                                    const unsigned long long* __restrict__ offsets,
                                                    const unsigned long long* __restrict__ qstage,
                                                    const dts_result* __restrict__ stage,
                                                    unsigned long long stage_n,
                                                    dts_result* __restrict__ out,
                                                    unsigned long long cap) {
    (void)stage_n;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t q0 = (blockIdx.x * 256 + threadIdx.x) & ~31u;
    if (q0 >= nq) return;
    const uint32_t q = q0 + lane;
    uint32_t c = 0;
    unsigned long long o = 0, sp = NONE;
    if (q < nq) {                             // three independent coalesced loads
        c = counts[q];
        sp = qstage[q];                       // (stale for c == 0: not used)
        o = offsets[q];
        if (c == 0 || sp == NONE) c = 0;
    }
    uint32_t inc = c;                         // staged records of lanes <= this one
#pragma unroll
    for (int k = 1; k < 32; k <<= 1) {
        const uint32_t u = __shfl_up_sync(0xffffffffu, inc, k);
        if (lane >= (uint32_t)k) inc += u;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
    for (uint32_t k0 = 0; k0 < total; k0 += 32) {
        const uint32_t k = k0 + lane;
        int src = 0;                          // the first lane whose records reach past k
#pragma unroll
        for (int step = 16; step; step >>= 1) {
            const uint32_t e = __shfl_sync(0xffffffffu, inc, src + step - 1);
            src += e <= k ? step : 0;
        }
        const uint32_t ex = __shfl_sync(0xffffffffu, inc - c, src);
        const unsigned long long os = __shfl_sync(0xffffffffu, o, src);
        const unsigned long long ss = __shfl_sync(0xffffffffu, sp, src);
        const unsigned long long j = os + (k - ex);
        DTS_DCHECK(k >= total || (k >= ex && ss != NONE && ss + (k - ex) < stage_n));
        if (k < total && j < cap) out[j] = stage[ss + (k - ex)];
    }
}

// ------------------------------- spilled tiles on an index with outliers
// Spilled records of the OUT pass 1 carry sorted positions: each is resolved
// to its entry id, and a hit on a copy that is not its query's canonical copy
// is dropped (query_id = DROPPED) and taken off the query's count.  The
// query's stencil is rebuilt from its row (make_stencil is a pure function of
// the query and the index, so it is the one pass 1 used).  Before the scan.
constexpr uint32_t DROPPED = 0xffffffffu;
__global__ void __launch_bounds__(128) k_spill_filter(const TileArgs a, unsigned long long n,
                                                     uint2* __restrict__ sp) {
    const OutlierArgs oa{a.out, a.soa, a.bin_t0min, a.bin_t1max};
    for (unsigned long long k = (unsigned long long)blockIdx.x * 128 + threadIdx.x; k < n;
         k += (unsigned long long)gridDim.x * 128) {
        const uint2 r = sp[k];                        // (query id, sorted position)
        const uint32_t p = r.y;
        if (is_copy(a.out, p)) {
            QState q{};
            double qlo[3], qhi[3];
            const bool live = load_query(a.Q, r.x, q, qlo, qhi);
            const Stencil st = make_stencil(a.g, q, qlo, qhi, a.d, live, a.bin_start,
                                            a.bin_t0min, a.bin_t1max, a.method, a.sb);
            QStencil qs;
            qs.lb = st.lb; qs.hb = st.hb;
            qs.mode = st.mode; qs.rind = st.rind;
            for (int ax = 0; ax < 3; ++ax) { qs.clo[ax] = st.clo[ax]; qs.cn[ax] = st.cn[ax]; }
            qs.rstart = st.rstart; qs.rcnt = st.rcnt;
            if (!outlier_canonical(&oa, &a.g, &qs, q.t0, q.t1, p)) {
                atomicSub(&a.counts[r.x], 1u);
                sp[k].x = DROPPED;
                continue;
            }
        }
        sp[k].y = __ldg(a.soa.eid + p);
    }
}

// The largest count among the spilled tiles' queries (after k_spill_filter).
__global__ void __launch_bounds__(128) k_spill_max(const uint32_t* __restrict__ tiles,
                                                  uint32_t ntl, uint32_t tq,
                                                  const uint32_t* __restrict__ order,
                                                  uint32_t nq, const uint32_t* __restrict__ counts,
                                                  Counters* __restrict__ ctr) {
    const uint32_t i = blockIdx.x * 128 + threadIdx.x;
    if (i >= ntl * tq) return;
    const uint32_t sp = tiles[i / tq] * tq + i % tq;
    if (sp >= nq) return;
    const uint32_t c = counts[order[sp]];
    if (c) atomicMax(&ctr->max_count, c);
}

// ------------------------------------------- spilled tiles: place + sort
// The spilled records: the first spill buffer, then the re-run's (index
// space [0, na) then [na, na + nb)).
struct SpillSrc {                       // the spilled intervals; the ids come with the keys
    const double2* a;
    unsigned long long na;
    const double2* b;
    // the record of spill index i with entry id e
    __device__ __forceinline__ dts_result at(uint32_t i, uint32_t e) const {
        const double2 t = i < na ? a[i] : b[i - na];
        dts_result r;
        r.query_id = 0;
        r.entry_id = e;
        r.t_start = t.x;
        r.t_end = t.y;
        return r;
    }
};

// Each live spilled record's key (entry id << 32 | its spill index) goes to
// its query's segment [offsets[q], offsets[q] + counts[q]) of `rkeys`, in
// arrival order: one atomic per (warp, query) group (__match_any_sync), not
// per record.  Records of queries whose tile was re-run (cover[q] != 0) are
// stale and skipped, and so are records the outlier filter dropped.  (Keys,
// 8 bytes, instead of the 24-byte records: the sorts read them contiguously
// and gather each record once, from the spill buffer.)
__global__ void __launch_bounds__(256) k_spill_place(const uint2* __restrict__ sp,
                                                    unsigned long long n, uint32_t base_idx,
                                                    const uint32_t* __restrict__ cover,
                                                    const unsigned long long* __restrict__ offsets,
                                                    uint32_t* __restrict__ cursor,
                                                    unsigned long long* __restrict__ rkeys) {
    const unsigned long long k = (unsigned long long)blockIdx.x * 256 + threadIdx.x;
    const int lane = threadIdx.x & 31;
    uint32_t q = 0xffffffffu, e = 0;
    bool live = k < n;
    if (live) {
        const uint2 qe = sp[k];                                    // (query_id, entry_id)
        q = qe.x;
        e = qe.y;
        if (q == DROPPED || (cover && cover[q])) live = false;
    }
    if (!live) q = 0xffffffffu;
    const uint32_t grp = __match_any_sync(0xffffffffu, q);
    if (!live) return;
    const int leader = __ffs(grp) - 1;
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(&cursor[q], (uint32_t)__popc(grp));
    base = __shfl_sync(grp, base, leader);
    DTS_DCHECK(offsets[q] + base + (uint32_t)__popc(grp) <= offsets[q + 1]);
    rkeys[offsets[q] + base + __popc(grp & ((1u << lane) - 1u))] =
        ((unsigned long long)e << 32) | (uint32_t)(base_idx + k);
}

// Spilled queries' segments of `raw` sorted by entry id into the output,
// by size: a warp per query up to SEGW_CAP records (an LSD radix sort of the
// entry id bits in shared memory; it visits every listed slot and queues the
// longer ones), a 256-thread CTA bitonic sort up to SEG_CAP, and a
// device-wide radix sort beyond (bigc).  The records are gathered into the
// output in entry id order with the reported query id (canonical; equal
// caller ids keep an unspecified order).  Measured (C2 at d = 8, 100 k
// queries of 342 records on average): one 256-thread CTA bitonic sort per
// query 1.91 ms; a warp bitonic sort per query 1.7 ms (O(n log^2 n) compare
// steps are the cost, not memory); S2 at d = 1 (8,400 per query): CTA
// bitonic sorts up to 16,384 records lost to the device-wide radix sort
// (canonicalisation 44 ms vs 39).
constexpr int SEGW_CAP = 512;
constexpr int SEG_MID = 4096;                  // k_seg_bucket<512, 8>: 4 CTAs per SM
constexpr int SEG_MID2 = 8192;                 // k_seg_bucket<512, 16>: 2 CTAs per SM
constexpr int SEG_CAP = 16384;                 // k_seg_bucket<1024, 16>: 1 CTA per SM

// A segment's (entry id << 32 | spill index) keys into shared memory, and
// the records gathered in key order into the output: UNR independent loads
// in flight per thread (a plain loop waits for each load before its store).
template <int UNR>
__device__ __forceinline__ void seg_keys_load(unsigned long long* key,
                                              const unsigned long long* rk, uint32_t c,
                                              uint32_t t, uint32_t nt) {
    for (uint32_t b = t; b < c; b += nt * UNR) {
        unsigned long long e[UNR];
#pragma unroll
        for (int j = 0; j < UNR; ++j) {
            const uint32_t i = b + (uint32_t)j * nt;
            e[j] = i < c ? rk[i] : 0ull;
        }
#pragma unroll
        for (int j = 0; j < UNR; ++j) {
            const uint32_t i = b + (uint32_t)j * nt;
            if (i < c) key[i] = e[j];
        }
    }
}

template <int UNR>
__device__ __forceinline__ void seg_gather(const unsigned long long* key, const SpillSrc& src,
                                           uint32_t c, uint32_t qrep, dts_result* out, uint32_t t,
                                           uint32_t nt) {
    for (uint32_t b = t; b < c; b += nt * UNR) {
        dts_result r[UNR];
#pragma unroll
        for (int j = 0; j < UNR; ++j) {
            const uint32_t i = b + (uint32_t)j * nt;
            if (i < c) r[j] = src.at((uint32_t)(key[i] & 0xffffffffull), (uint32_t)(key[i] >> 32));
        }
#pragma unroll
        for (int j = 0; j < UNR; ++j) {
            const uint32_t i = b + (uint32_t)j * nt;
            if (i < c) {
                r[j].query_id = qrep;
                out[i] = r[j];
            }
        }
    }
}

struct SegWarpSmem {
    unsigned long long buf[2][SEGW_CAP];
    uint32_t cnt[256];
};

__global__ void __launch_bounds__(128) k_seg_sort_warp(const uint32_t* __restrict__ tiles,
                                                      uint32_t nslots, uint32_t tq,
                                                      const uint32_t* __restrict__ order,
                                                      uint32_t nq,
                                                      const uint32_t* __restrict__ counts,
                                                      const unsigned long long* __restrict__ offsets,
                                                      const unsigned long long* __restrict__ rkeys,
                                                      const SpillSrc src,
                                                      const uint32_t* __restrict__ qmap,
                                                      uint32_t qid_base, int eb,
                                                      dts_result* __restrict__ out,
                                                      uint32_t* __restrict__ lists,   // 4 x lstride
                                                      size_t lstride,
                                                      uint32_t* __restrict__ bigc,
                                                      Counters* __restrict__ ctr) {
    __shared__ SegWarpSmem SWS[4];
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t w = blockIdx.x * 4 + warp;
    if (w >= nslots) return;
    const uint32_t sp = tiles[w / tq] * tq + w % tq;
    if (sp >= nq) return;
    const uint32_t q = order[sp];
    const uint32_t c = counts[q];
    if (c == 0) return;
    if (c > (uint32_t)SEGW_CAP) {
        if (lane == 0) {
            if (c <= (uint32_t)SEG_CAP) {
                const int k = c <= (uint32_t)SEG_MID ? 0 : (c <= (uint32_t)SEG_MID2 ? 1 : 2);
                lists[(size_t)k * lstride + atomicAdd(&ctr->n_cls[k], 1u)] = q;
            } else {                              // listed in region 3 (k_big_split)
                lists[(size_t)3 * lstride + atomicAdd(&ctr->n_big, 1u)] = q;
            }
        }
        return;
    }
    SegWarpSmem& S = SWS[warp];
    const unsigned long long off = offsets[q];
    seg_keys_load<8>(S.buf[0], rkeys + off, c, lane, 32);
    const uint32_t lt = (1u << lane) - 1u;
    int cur = 0;
    for (int sh = 32; sh < 32 + eb; sh += 8, cur ^= 1) {
        const unsigned long long* A = S.buf[cur];
        unsigned long long* B = S.buf[cur ^ 1];
#pragma unroll
        for (int j = 0; j < 8; ++j) S.cnt[lane * 8 + j] = 0;
        __syncwarp();
        for (uint32_t b0 = 0; b0 < c; b0 += 32) {           // digit histogram
            const uint32_t i = b0 + lane;
            if (i < c) atomicAdd(&S.cnt[(uint32_t)(A[i] >> sh) & 255u], 1u);
        }
        __syncwarp();
        {                                                   // exclusive scan, 8 per lane
            uint32_t v[8], tot = 0;
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] = S.cnt[lane * 8 + j]; tot += v[j]; }
            uint32_t inc = tot;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= (uint32_t)o) inc += u;
            }
            uint32_t run = inc - tot;
#pragma unroll
            for (int j = 0; j < 8; ++j) { S.cnt[lane * 8 + j] = run; run += v[j]; }
        }
        __syncwarp();
        for (uint32_t b0 = 0; b0 < c; b0 += 32) {           // stable scatter
            const uint32_t i = b0 + lane;
            const bool valid = i < c;
            const unsigned long long k = valid ? A[i] : 0ull;
            const uint32_t dig = (uint32_t)(k >> sh) & 255u;
            uint32_t peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
            for (int bit = 0; bit < 8; ++bit) {
                const uint32_t bal = __ballot_sync(0xffffffffu, (dig >> bit) & 1u);
                peers &= ((dig >> bit) & 1u) ? bal : ~bal;
            }
            const uint32_t base = valid ? S.cnt[dig] : 0u;
            __syncwarp();
            if (valid) {
                if (lane == 31u - __clz(peers)) S.cnt[dig] = base + __popc(peers);
                B[base + __popc(peers & lt)] = k;
            }
            __syncwarp();
        }
    }
    __syncwarp();
    const uint32_t qrep = qmap ? __ldg(qmap + q) : q + qid_base;
    seg_gather<4>(S.buf[cur], src, c, qrep, out + off, lane, 32);
}

// A segment to sort: `c` keys at key_base + off, sorted into out + off with
// the reported id of query q.  DESC: the i-th entry of a descriptor list
// (sub-segments of split long segments, k_big_split); else the listed
// query's whole segment.
struct SegDesc {
    const unsigned long long* off;
    const uint32_t* cnt;
    const uint32_t* q;
};
template <bool DESC>
__device__ __forceinline__ void seg_of(const uint32_t* list, const SegDesc& ds, uint32_t i,
                                       const uint32_t* counts,
                                       const unsigned long long* offsets, uint32_t& q, uint32_t& c,
                                       unsigned long long& off) {
    if (DESC) {
        q = ds.q[i];
        c = ds.cnt[i];
        off = ds.off[i];
    } else {
        q = list[i];
        c = counts[q];
        off = offsets[q];
    }
}

// One CTA of SEGC_T threads per listed query (SEGW_CAP < count <= SEGC_T *
// ITEMS): an LSD radix sort of the (entry id << 32 | slot) keys over the
// entry id bits, 8 bits per pass, the keys in one shared-memory buffer
// between passes.  Per pass a warp ranks its contiguous range of keys
// (ballot multisplit, ITEMS keys per lane kept in registers with their
// ranks), the per-warp digit counts are scanned across warps and digits,
// and every key is stored at its stable position (all keys are in
// registers by then, so the buffer is overwritten in place).
template <int SEGC_T, int ITEMS, int MINB, bool DESC = false>
__global__ void __launch_bounds__(SEGC_T, MINB) k_seg_radix(const uint32_t* __restrict__ list,
                                                        const uint32_t* __restrict__ counts,
                                                        const unsigned long long* __restrict__ offsets,
                                                        const unsigned long long* __restrict__ rkeys,
                                                      const SpillSrc src,
                                                        const uint32_t* __restrict__ qmap,
                                                        uint32_t qid_base, int eb,
                                                        dts_result* __restrict__ out,
                                                        const SegDesc ds) {
    constexpr int SEGC_W = SEGC_T / 32;
    extern __shared__ unsigned long long sbuf[];        // SEGC_T * ITEMS keys
    __shared__ uint32_t wcnt[SEGC_W][257];
    __shared__ uint32_t wtot[8];
    uint32_t q, c;
    unsigned long long off;
    seg_of<DESC>(list, ds, DESC ? list[blockIdx.x] : blockIdx.x, counts, offsets, q, c, off);
    // (non-DESC: seg_of reads list[blockIdx.x] as the query)
    const uint32_t t = threadIdx.x, lane = t & 31, warp = t >> 5;
    seg_keys_load<8>(sbuf, rkeys + off, c, t, SEGC_T);
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t wbase = warp * 32u * ITEMS;
    for (int sh = 32; sh < 32 + eb; sh += 8) {
        for (uint32_t j = lane; j < 257; j += 32) wcnt[warp][j] = 0;
        __syncthreads();
        unsigned long long k[ITEMS];
        uint32_t rk[ITEMS / 2];                      // two 16-bit ranks per word
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t p = wbase + (uint32_t)i * 32u + lane;
            const bool valid = p < c;
            k[i] = valid ? sbuf[p] : 0ull;
            const uint32_t dig = valid ? ((uint32_t)(k[i] >> sh) & 255u) : 256u;
            uint32_t peers = 0xffffffffu;
#pragma unroll
            for (int b = 0; b < 9; ++b) {
                const uint32_t bal = __ballot_sync(0xffffffffu, (dig >> b) & 1u);
                peers &= ((dig >> b) & 1u) ? bal : ~bal;
            }
            const uint32_t base = wcnt[warp][dig];
            __syncwarp();
            if (lane == 31u - __clz(peers)) wcnt[warp][dig] = base + __popc(peers);
            const uint32_t r = base + __popc(peers & lt);
            rk[i / 2] = (i & 1) ? (rk[i / 2] | (r << 16)) : r;
            __syncwarp();
        }
        __syncthreads();
        // digit d (thread d < 256): counts of the warps before -> per-warp
        // base, then an exclusive scan of the digit totals
        uint32_t tot = 0;
        if (t < 256) {
#pragma unroll
            for (int w = 0; w < SEGC_W; ++w) {
                const uint32_t x = wcnt[w][t];
                wcnt[w][t] = tot;
                tot += x;
            }
        }
        uint32_t inc = tot;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= (uint32_t)o) inc += u;
        }
        if (t < 256 && lane == 31) wtot[warp] = inc;
        __syncthreads();
        if (t < 256) {
            uint32_t pre = inc - tot;
            for (uint32_t w = 0; w < warp; ++w) pre += wtot[w];
#pragma unroll
            for (int w = 0; w < SEGC_W; ++w) wcnt[w][t] += pre;
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t p = wbase + (uint32_t)i * 32u + lane;
            if (p < c)
                sbuf[wcnt[warp][(uint32_t)(k[i] >> sh) & 255u] + ((rk[i / 2] >> (16 * (i & 1))) & 0xffffu)] = k[i];
        }
        __syncthreads();
    }
    const uint32_t qrep = qmap ? __ldg(qmap + q) : q + qid_base;
    seg_gather<4>(sbuf, src, c, qrep, out + off, t, SEGC_T);
}

// One CTA of T threads per listed query (SEGW_CAP < count <= CAP): a
// counting sort on the high bits of (entry id - the segment's least id)
// into about one bucket per record (shared-memory atomics, no ranking
// ballots), then an insertion sort of each bucket by one thread.  A segment
// whose ids cluster (a bucket over SEGB_MAX records) is sorted by the
// ballot-ranked radix sort instead (queued on skew_list).  Measured on S2 at
// d = 1 (292 M records in segments of 4,097-16,384): the radix sort's
// ballot multisplit (9 ballots per key per 8-bit pass) took 13.0 ms.
constexpr int SEGB_MAX = 32;

template <int T, int ITEMS, int MINB, bool DESC = false>
__global__ void __launch_bounds__(T, MINB) k_seg_bucket(const uint32_t* __restrict__ list,
                                                       const uint32_t* __restrict__ counts,
                                                       const unsigned long long* __restrict__ offsets,
                                                       const unsigned long long* __restrict__ rkeys,
                                                      const SpillSrc src,
                                                       const uint32_t* __restrict__ qmap,
                                                       uint32_t qid_base,
                                                       dts_result* __restrict__ out,
                                                       uint32_t* __restrict__ skew_list,
                                                       Counters* __restrict__ ctr,
                                                       const SegDesc ds) {
    constexpr uint32_t CAP = (uint32_t)T * ITEMS;
    extern __shared__ unsigned long long bbuf[];        // CAP keys, then CAP bucket counters
    uint32_t* cnt = reinterpret_cast<uint32_t*>(bbuf + CAP);
    __shared__ uint32_t s_min, s_max, s_bmax, s_wsum[T / 32];
    // (DESC: blockIdx.x is the descriptor; skewed ones are listed by index)
    uint32_t q, c;
    unsigned long long off;
    seg_of<DESC>(list, ds, blockIdx.x, counts, offsets, q, c, off);
    const unsigned long long* rk = rkeys + off;
    const uint32_t t = threadIdx.x, lane = t & 31, warp = t >> 5;
    if (t == 0) { s_min = ~0u; s_max = 0u; s_bmax = 0u; }
    // ---- the segment's keys (entry id << 32 | spill index), held in
    //      registers (slot t + j*T), and the range of their ids
    unsigned long long kk[ITEMS];
    uint32_t mn = ~0u, mx = 0u;
#pragma unroll
    for (int j = 0; j < ITEMS; ++j) {
        const uint32_t i = t + (uint32_t)j * T;
        kk[j] = i < c ? rk[i] : 0ull;
    }
#pragma unroll
    for (int j = 0; j < ITEMS; ++j) {
        const uint32_t e = (uint32_t)(kk[j] >> 32);
        if (t + (uint32_t)j * T < c) { mn = min(mn, e); mx = max(mx, e); }
    }
    mn = __reduce_min_sync(0xffffffffu, mn);
    mx = __reduce_max_sync(0xffffffffu, mx);
    uint32_t nb = 32;
    while (nb < c) nb <<= 1;
    for (uint32_t i = t; i < nb; i += T) cnt[i] = 0;
    __syncthreads();
    if (lane == 0) { atomicMin(&s_min, mn); atomicMax(&s_max, mx); }
    __syncthreads();
    mn = s_min;
    const uint32_t span = s_max - mn;
    const int sbits = span ? 32 - __clz(span) : 0;
    const int lnb = 31 - __clz(nb);
    const int sh = sbits > lnb ? sbits - lnb : 0;
    // ---- bucket counts
#pragma unroll
    for (int j = 0; j < ITEMS; ++j)
        if (t + (uint32_t)j * T < c) atomicAdd(&cnt[((uint32_t)(kk[j] >> 32) - mn) >> sh], 1u);
    __syncthreads();
    // ---- exclusive scan of the counters (nb / T per thread, consecutive)
    const uint32_t per = (nb + T - 1) / T, b0 = t * per;
    uint32_t sum = 0, bmax = 0;
    for (uint32_t j = 0; j < per; ++j) {
        if (b0 + j < nb) { const uint32_t x = cnt[b0 + j]; sum += x; bmax = max(bmax, x); }
    }
    bmax = __reduce_max_sync(0xffffffffu, bmax);
    uint32_t inc = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t u = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= (uint32_t)o) inc += u;
    }
    if (lane == 31) s_wsum[warp] = inc;
    if (lane == 0) atomicMax(&s_bmax, bmax);
    __syncthreads();
    if (s_bmax > (uint32_t)SEGB_MAX) {              // clustered ids: the radix sort
        if (t == 0) {
            if (DESC) skew_list[atomicAdd(&ctr->n_dskew, 1u)] = blockIdx.x;
            else skew_list[atomicAdd(&ctr->n_skew, 1u)] = q;
        }
        return;
    }
    uint32_t run = inc - sum;
    for (uint32_t w = 0; w < warp; ++w) run += s_wsum[w];
    for (uint32_t j = 0; j < per; ++j) {
        if (b0 + j < nb) { const uint32_t x = cnt[b0 + j]; cnt[b0 + j] = run; run += x; }
    }
    __syncthreads();
    // ---- scatter into the buckets (cnt[b] ends at the end of bucket b)
#pragma unroll
    for (int j = 0; j < ITEMS; ++j) {
        const uint32_t i = t + (uint32_t)j * T;
        if (i < c) bbuf[atomicAdd(&cnt[((uint32_t)(kk[j] >> 32) - mn) >> sh], 1u)] = kk[j];
    }
    __syncthreads();
    // ---- each bucket sorted by one thread (insertion sort, <= SEGB_MAX keys)
    for (uint32_t b = t; b < nb; b += T) {
        const uint32_t lo = b ? cnt[b - 1] : 0u, hi = cnt[b];
        for (uint32_t i = lo + 1; i < hi; ++i) {
            const unsigned long long k = bbuf[i];
            uint32_t j = i;
            while (j > lo && bbuf[j - 1] > k) { bbuf[j] = bbuf[j - 1]; --j; }
            bbuf[j] = k;
        }
    }
    __syncthreads();
    const uint32_t qrep = qmap ? __ldg(qmap + q) : q + qid_base;
    seg_gather<4>(bbuf, src, c, qrep, out + off, t, T);
}

// Segments longer than SEG_CAP, one CTA each: the keys are split into
// B = ceil(c / SEG_SPLIT) equal-width ranges of (entry id - the segment's
// least id) -- ordered ranges, so sorting each range in place sorts the
// segment -- written to `rk2` at the segment's offsets, and one descriptor
// per non-empty range is listed for k_seg_bucket<DESC>.  A segment whose
// ranges do not all fit a CTA sort (ids clustered) is left to the
// device-wide sort (bigc[q] = c).
constexpr int SEG_SPLIT = 8192;
constexpr int SPLIT_MAXB = 256;
__global__ void __launch_bounds__(256) k_big_split(const uint32_t* __restrict__ list,
                                                  const uint32_t* __restrict__ counts,
                                                  const unsigned long long* __restrict__ offsets,
                                                  const unsigned long long* __restrict__ rkeys,
                                                  unsigned long long* __restrict__ rk2,
                                                  uint32_t* __restrict__ bigc,
                                                  unsigned long long* __restrict__ d_off,
                                                  uint32_t* __restrict__ d_cnt,
                                                  uint32_t* __restrict__ d_q,
                                                  Counters* __restrict__ ctr) {
    __shared__ uint32_t s_min, s_max, s_ok, cnt[SPLIT_MAXB], base[SPLIT_MAXB];
    const uint32_t q = list[blockIdx.x];
    const uint32_t c = counts[q];
    const unsigned long long off = offsets[q];
    const unsigned long long* rk = rkeys + off;
    const uint32_t t = threadIdx.x;
    uint32_t B = (c + SEG_SPLIT - 1) / SEG_SPLIT;
    if (t == 0) { s_min = ~0u; s_max = 0u; s_ok = 1u; }
    for (uint32_t j = t; j < SPLIT_MAXB; j += 256) cnt[j] = 0;
    __syncthreads();
    if (B > (uint32_t)SPLIT_MAXB) {                  // beyond the split: device sort
        if (t == 0) {
            bigc[q] = c;
            atomicAdd(&ctr->n_bigfb, 1u);
        }
        return;
    }
    uint32_t mn = ~0u, mx = 0u;
    for (uint32_t i = t; i < c; i += 256) {
        const uint32_t e = (uint32_t)(rk[i] >> 32);
        mn = min(mn, e);
        mx = max(mx, e);
    }
    mn = __reduce_min_sync(0xffffffffu, mn);
    mx = __reduce_max_sync(0xffffffffu, mx);
    if ((t & 31) == 0) { atomicMin(&s_min, mn); atomicMax(&s_max, mx); }
    __syncthreads();
    mn = s_min;
    const unsigned long long span = (unsigned long long)(s_max - mn) + 1ull;
    auto bucket = [&](unsigned long long k) {
        return (uint32_t)(((unsigned long long)((uint32_t)(k >> 32) - mn) * B) / span);
    };
    for (uint32_t i = t; i < c; i += 256) atomicAdd(&cnt[bucket(rk[i])], 1u);
    __syncthreads();
    if (t == 0) {
        uint32_t run = 0;
        for (uint32_t b = 0; b < B; ++b) {
            if (cnt[b] > (uint32_t)SEG_CAP) s_ok = 0u;
            base[b] = run;
            run += cnt[b];
        }
    }
    __syncthreads();
    if (!s_ok) {                                     // clustered ids: device sort
        if (t == 0) {
            bigc[q] = c;
            atomicAdd(&ctr->n_bigfb, 1u);
        }
        return;
    }
    if (t < B && cnt[t]) {
        const uint32_t k = atomicAdd(&ctr->n_desc, 1u);
        d_off[k] = off + base[t];
        d_cnt[k] = cnt[t];
        d_q[k] = q;
    }
    __syncthreads();
    for (uint32_t i = t; i < c; i += 256) {
        const unsigned long long k = rk[i];
        const uint32_t pos = atomicAdd(&base[bucket(k)], 1u);
        DTS_DCHECK(bucket(k) < B && pos < c);
        rk2[off + pos] = k;
    }
}

// Segments longer than SEG_CAP: one device-wide keys-only radix sort of
// packed keys (query << (eb + sb) | entry id << sb | slot in segment) on the
// (query, entry id) bits; the slot rides in the low bits.  One warp per query.
__global__ void __launch_bounds__(256) k_big_keys(uint32_t nq, const uint32_t* __restrict__ bigc,
                                                 const unsigned long long* __restrict__ bigoff,
                                                 const unsigned long long* __restrict__ offsets,
                                                 const unsigned long long* __restrict__ rkeys,
                                                 int eb, int sb,
                                                 unsigned long long* __restrict__ keys) {
    const uint32_t warp = (blockIdx.x * 256 + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (warp >= nq) return;
    const uint32_t c = bigc[warp];
    if (!c) return;
    const unsigned long long o = offsets[warp], b = bigoff[warp];
    const unsigned long long qk = (unsigned long long)warp << (eb + sb);
    for (uint32_t i = lane; i < c; i += 32)
        keys[b + i] = qk | ((rkeys[o + i] >> 32) << sb) | i;
}

// out[k-th place of its segment] = the spilled record of its segment's key
// at the slot of sorted element k, with the reported query id
__global__ void __launch_bounds__(256) k_big_place(const unsigned long long* __restrict__ keys,
                                                  unsigned long long n, int eb, int sb,
                                                  const unsigned long long* __restrict__ bigoff,
                                                  const unsigned long long* __restrict__ offsets,
                                                  const unsigned long long* __restrict__ rkeys,
                                                  const SpillSrc src,
                                                  const uint32_t* __restrict__ qmap,
                                                  uint32_t qid_base,
                                                  dts_result* __restrict__ out) {
    const unsigned long long k = (unsigned long long)blockIdx.x * 256 + threadIdx.x;
    if (k >= n) return;
    const unsigned long long key = keys[k];
    const uint32_t q = (uint32_t)(key >> (eb + sb));
    const unsigned long long slot = key & ((1ull << sb) - 1ull);
    const unsigned long long rkey = rkeys[offsets[q] + slot];
    dts_result r = src.at((uint32_t)(rkey & 0xffffffffull), (uint32_t)(rkey >> 32));
    r.query_id = qmap ? __ldg(qmap + q) : q + qid_base;
    out[offsets[q] + (k - bigoff[q])] = r;
}
