/*
 * oracle.c -- plain, slow, obviously correct CPU reference of the distance
 * threshold search of Gowanlock & Casanova (PAPER.md, dblp conf/ipps/GowanlockC15).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load or call this code.
 * The product library (libdts.so) never links it, and it shares no code,
 * header, table or constant with the CUDA path.
 *
 * What it computes (§III "Problem statement"): for a query set Q
 * and an entry database D of 4-D line segments (1 temporal + 3 spatial
 * dimensions), every (q, l, [t_s, t_e]) such that q and l are within distance d
 * of each other during [t_s, t_e].  The paper's kernels find candidates with an
 * index and then refine each candidate with compare() (Alg. 1 l.14 P:L64,
 * Alg. 3 l.12 P:L112); an index only prunes, so the oracle is the plain
 * definition: compare() applied to every one of the |Q| x |D| pairs, in fp64
 * (the paper states no precision), single threaded, compiled
 * with -O2 -ffp-contract=off.
 *
 * compare() is never written out in the paper; the steps below
 * are the readings c1-c4 of DESIGN.md §"Readings":
 *   1. temporal overlap  ts = max(t_start), te = min(t_end); none unless ts < te
 *      (strict overlap, reading c2);
 *   2. positions by linear interpolation in time along each segment
 *      (segments are straight lines between their spatiotemporal endpoints,
 *      P:L32);
 *   3. relative position A at ts, B at te, V = B - A  (relative motion of two
 *      linear motions is linear: Delta(tau) = A + tau V, tau in [0,1]);
 *   4. |Delta(tau)|^2 - d^2 = a tau^2 + 2 beta tau + c with a = V.V,
 *      beta = A.V, c = A.A - d^2;
 *   5. the set where it is <= 0 (closed inequality, reading c3), intersected
 *      with [0,1]; roots by the textbook quadratic formula in its
 *      cancellation-free form (q = -(beta + sign(beta) sqrt(disc)),
 *      roots q/a and c/q);
 *   6. map [lo,hi] back to absolute time.
 * Results are produced in (query id, entry id) ascending order (reading c7)
 * because the loops run that way.
 *
 * Parity pins for every function here are in tests/test_oracle.py; none is
 * "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* One segment: spatiotemporal start point and end point. */
typedef struct {
    double t_start, x_start, y_start, z_start;
    double t_end, x_end, y_end, z_end;
} oracle_segment;

/* One result triple (q, l, [t_s, t_e]). */
typedef struct {
    uint32_t query_id;
    uint32_t entry_id;
    double t_start;
    double t_end;
} oracle_result;

/* Step 2: position of segment s at time t, t in [s.t_start, s.t_end],
 * s.t_end > s.t_start.  f = (t - t_start) / (t_end - t_start),
 * P(t) = (1 - f) P_start + f P_end  (exact at f = 0 and f = 1). */
static void position_at(const oracle_segment *s, double t, double p[3])
{
    double f = (t - s->t_start) / (s->t_end - s->t_start);
    p[0] = (1.0 - f) * s->x_start + f * s->x_end;
    p[1] = (1.0 - f) * s->y_start + f * s->y_end;
    p[2] = (1.0 - f) * s->z_start + f * s->z_end;
}

/* Steps 1-4 shared by compare() and the tie-band distance: returns 0 when the
 * segments do not overlap strictly in time. */
static int relative_motion(const oracle_segment *q, const oracle_segment *l,
                           double *ts, double *te, double A[3], double V[3])
{
    double pq[3], pl[3], B[3];
    *ts = q->t_start > l->t_start ? q->t_start : l->t_start;   /* max */
    *te = q->t_end < l->t_end ? q->t_end : l->t_end;           /* min */
    if (!(*ts < *te))
        return 0;
    position_at(q, *ts, pq);
    position_at(l, *ts, pl);
    A[0] = pl[0] - pq[0]; A[1] = pl[1] - pq[1]; A[2] = pl[2] - pq[2];
    position_at(q, *te, pq);
    position_at(l, *te, pl);
    B[0] = pl[0] - pq[0]; B[1] = pl[1] - pq[1]; B[2] = pl[2] - pq[2];
    V[0] = B[0] - A[0]; V[1] = B[1] - A[1]; V[2] = B[2] - A[2];
    return 1;
}

/* compare(D[e], Q[q]) of Alg. 1 l.14 / Alg. 3 l.12.
 * Returns 1 and the interval during which |P_l(t) - P_q(t)| <= d, else 0. */
int oracle_compare(const oracle_segment *q, const oracle_segment *l, double d,
                   double *t_s, double *t_e)
{
    double ts, te, A[3], V[3];
    if (!relative_motion(q, l, &ts, &te, A, V))
        return 0;
    double a = V[0] * V[0] + V[1] * V[1] + V[2] * V[2];
    double beta = A[0] * V[0] + A[1] * V[1] + A[2] * V[2];
    double c = A[0] * A[0] + A[1] * A[1] + A[2] * A[2] - d * d;
    double lo, hi;
    if (a == 0.0) {                       /* no relative motion */
        if (!(c <= 0.0))
            return 0;
        lo = 0.0; hi = 1.0;
    } else {
        double disc = beta * beta - a * c;
        if (disc < 0.0)
            return 0;
        double r = sqrt(disc);
        double qq = -(beta + (beta >= 0.0 ? r : -r));
        double tau1, tau2;
        if (qq == 0.0) {                  /* beta = 0 and disc = 0: double root */
            tau1 = tau2 = -beta / a;
        } else {
            double x1 = qq / a, x2 = c / qq;
            tau1 = x1 < x2 ? x1 : x2;
            tau2 = x1 < x2 ? x2 : x1;
        }
        lo = tau1 > 0.0 ? tau1 : 0.0;
        hi = tau2 < 1.0 ? tau2 : 1.0;
        if (lo > hi)
            return 0;
    }
    *t_s = (1.0 - lo) * ts + lo * te;
    *t_e = (1.0 - hi) * ts + hi * te;
    return 1;
}

/* Minimum distance between q and l over their strict temporal overlap
 * (the quantity whose closeness to d defines the parity tie band, reading
 * c11).  tau* = clamp(-beta/a, 0, 1), d_min = |A + tau* V|.  Returns 0 when
 * the segments do not overlap strictly in time. */
int oracle_dmin(const oracle_segment *q, const oracle_segment *l, double *dmin)
{
    double ts, te, A[3], V[3];
    if (!relative_motion(q, l, &ts, &te, A, V))
        return 0;
    double a = V[0] * V[0] + V[1] * V[1] + V[2] * V[2];
    double beta = A[0] * V[0] + A[1] * V[1] + A[2] * V[2];
    double tau = 0.0;
    if (a > 0.0) {
        tau = -beta / a;
        if (tau < 0.0) tau = 0.0;
        if (tau > 1.0) tau = 1.0;
    }
    double x = A[0] + tau * V[0], y = A[1] + tau * V[1], z = A[2] + tau * V[2];
    *dmin = sqrt(x * x + y * y + z * z);
    return 1;
}

/* Brute-force search of queries [q_begin, q_end) against all of D:
 * compare() on every pair, results appended in (query, entry) order.
 * Output buffer is malloc'd; free with oracle_free().  Returns 0 on success,
 * -1 on allocation failure. */
int oracle_search(const oracle_segment *D, uint64_t n,
                  const oracle_segment *Q, uint64_t q_begin, uint64_t q_end,
                  double d, oracle_result **out, uint64_t *count)
{
    uint64_t cap = 1024, cnt = 0;
    oracle_result *buf = (oracle_result *)malloc(cap * sizeof(oracle_result));
    if (!buf)
        return -1;
    for (uint64_t qi = q_begin; qi < q_end; ++qi) {
        for (uint64_t li = 0; li < n; ++li) {
            double ts, te;
            if (oracle_compare(&Q[qi], &D[li], d, &ts, &te)) {
                if (cnt == cap) {
                    cap *= 2;
                    oracle_result *nb = (oracle_result *)realloc(buf, cap * sizeof(oracle_result));
                    if (!nb) { free(buf); return -1; }
                    buf = nb;
                }
                buf[cnt].query_id = (uint32_t)qi;
                buf[cnt].entry_id = (uint32_t)li;
                buf[cnt].t_start = ts;
                buf[cnt].t_end = te;
                ++cnt;
            }
        }
    }
    *out = buf;
    *count = cnt;
    return 0;
}

/* d_min for a list of (query id, entry id) pairs; writes NAN when the pair
 * does not overlap strictly in time. */
void oracle_dmin_pairs(const oracle_segment *D, const oracle_segment *Q,
                       const uint32_t *qids, const uint32_t *eids, uint64_t m,
                       double *out)
{
    for (uint64_t i = 0; i < m; ++i) {
        double v;
        out[i] = oracle_dmin(&Q[qids[i]], &D[eids[i]], &v) ? v : NAN;
    }
}

/* compare() for a list of pairs (used by invariance tests). */
void oracle_compare_pairs(const oracle_segment *D, const oracle_segment *Q,
                          const uint32_t *qids, const uint32_t *eids, uint64_t m,
                          double d, int32_t *hit, double *ts, double *te)
{
    for (uint64_t i = 0; i < m; ++i) {
        double a = NAN, b = NAN;
        hit[i] = oracle_compare(&Q[qids[i]], &D[eids[i]], d, &a, &b);
        ts[i] = a;
        te[i] = b;
    }
}

void oracle_free(void *p) { free(p); }
