/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what SMiLer's Search
 * Step computes (Zhou & Tung, SIGMOD'15, /root/reference/PAPER.md, cited as
 * P:<line>).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or execute it.  It shares no
 * code, header, table or constant with the CUDA path under
 * paper_conf_sigmod_zhout15_b200/ and never includes anything from there.
 *
 * Build: gcc -O2 -fno-fast-math -ffp-contract=off -fopenmp -shared -fPIC
 * (-ffp-contract=off so that the only fused multiply-add in the f32 DTW is
 * the explicit fmaf of reading R16.)
 *
 * Readings of the paper used here:
 *   R1  dist(a,b) = (a-b)^2, no final square root.
 *   R2  segment C_{t,d} = c[t .. t+d), 0-based, d points; its id is t.
 *   R3  envelopes are clipped to the series (or MQ) range.
 *   R4  band >= 1 -> absolute rho; band < 1 -> rho_i = floor(band*d_i).
 *       Lower-bound envelopes use rho_env = max_i rho_i (passed in).
 *   R6  a candidate with no full disjoint window has LB_w = 0.
 *   R11 ties ordered by (dist, t): lowest t first.
 *   R12 fewer than k candidates -> pad with id -1 and dist "infinity".
 *   R16 f32 DTW cell = fmaf(q-c, q-c, min3) in float.
 *   R19 SW_b = MQ[D-w-b .. D-b)   (sliding windows numbered right to left).
 *   R20 LB_EQ of every item query uses the master query's envelope.
 *
 * Parity status of each function: see the "pins" listed in DESIGN.md and
 * tests/test_oracle_pins.py.  Every function below is pinned.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORC_INF_I64 (INT64_MAX / 4)

/* ------------------------------------------------------------------------ */
/* Envelope, Def. B.1 / Eq. 25:                                 */
/*   U_i = max_{-rho<=r<=rho} c_{i+r},  L_i = min_{-rho<=r<=rho} c_{i+r}      */
/* clipped to [0, n) (R3).                                                    */
/* ------------------------------------------------------------------------ */
void orc_envelope_i64(const int64_t *x, int64_t n, int64_t rho, int64_t *U, int64_t *L)
{
    for (int64_t i = 0; i < n; i++) {
        int64_t lo = i - rho < 0 ? 0 : i - rho;
        int64_t hi = i + rho > n - 1 ? n - 1 : i + rho;
        int64_t mx = x[lo], mn = x[lo];
        for (int64_t j = lo; j <= hi; j++) {
            if (x[j] > mx) mx = x[j];
            if (x[j] < mn) mn = x[j];
        }
        U[i] = mx;
        L[i] = mn;
    }
}

void orc_envelope_f64(const double *x, int64_t n, int64_t rho, double *U, double *L)
{
    for (int64_t i = 0; i < n; i++) {
        int64_t lo = i - rho < 0 ? 0 : i - rho;
        int64_t hi = i + rho > n - 1 ? n - 1 : i + rho;
        double mx = x[lo], mn = x[lo];
        for (int64_t j = lo; j <= hi; j++) {
            if (x[j] > mx) mx = x[j];
            if (x[j] < mn) mn = x[j];
        }
        U[i] = mx;
        L[i] = mn;
    }
}

/* ------------------------------------------------------------------------ */
/* Banded DTW, Eq. 21-24, full (d+1) x (d+1) matrix:           */
/*   g(0,0) = 0, g(i,0) = g(0,j) = inf                             (Eq. 22)  */
/*   g(i,j) = inf                               if |i-j| > rho     (Eq. 23)  */
/*   g(i,j) = dist(q_i, c_j) + min(g(i-1,j), g(i,j-1), g(i-1,j-1)) (Eq. 21)  */
/*   DTW    = g(d,d)                                               (Eq. 24)  */
/* q and c are 1-based in the paper; here q[i-1], c[j-1].                    */
/* ------------------------------------------------------------------------ */
static int64_t min3_i64(int64_t a, int64_t b, int64_t c)
{
    int64_t m = a < b ? a : b;
    return m < c ? m : c;
}

int64_t orc_dtw_i64(const int64_t *q, const int64_t *c, int d, int rho)
{
    int64_t *g = (int64_t *)malloc(sizeof(int64_t) * (size_t)(d + 1) * (size_t)(d + 1));
    for (int i = 0; i <= d; i++)
        for (int j = 0; j <= d; j++)
            g[i * (d + 1) + j] = ORC_INF_I64;
    g[0] = 0;
    for (int i = 1; i <= d; i++) {
        for (int j = 1; j <= d; j++) {
            if (abs(i - j) > rho) continue;                  /* Eq. 23 */
            int64_t diff = q[i - 1] - c[j - 1];
            int64_t m = min3_i64(g[(i - 1) * (d + 1) + j], g[i * (d + 1) + j - 1],
                                 g[(i - 1) * (d + 1) + j - 1]);
            if (m >= ORC_INF_I64) continue;                  /* unreachable cell */
            g[i * (d + 1) + j] = diff * diff + m;
        }
    }
    int64_t r = g[d * (d + 1) + d];
    free(g);
    return r;
}

static double min3_f64(double a, double b, double c)
{
    double m = a < b ? a : b;
    return m < c ? m : c;
}

double orc_dtw_f64(const double *q, const double *c, int d, int rho)
{
    double *g = (double *)malloc(sizeof(double) * (size_t)(d + 1) * (size_t)(d + 1));
    for (int i = 0; i <= d; i++)
        for (int j = 0; j <= d; j++)
            g[i * (d + 1) + j] = INFINITY;
    g[0] = 0.0;
    for (int i = 1; i <= d; i++) {
        for (int j = 1; j <= d; j++) {
            if (abs(i - j) > rho) continue;
            double diff = q[i - 1] - c[j - 1];
            double m = min3_f64(g[(i - 1) * (d + 1) + j], g[i * (d + 1) + j - 1],
                                g[(i - 1) * (d + 1) + j - 1]);
            g[i * (d + 1) + j] = diff * diff + m;
        }
    }
    double r = g[d * (d + 1) + d];
    free(g);
    return r;
}

/* f32 with the arithmetic pinned by reading R16: diff = q - c rounded to float,
 * cell = fmaf(diff, diff, min3).  Same recurrence as above. */
float orc_dtw_f32(const float *q, const float *c, int d, int rho)
{
    float *g = (float *)malloc(sizeof(float) * (size_t)(d + 1) * (size_t)(d + 1));
    for (int i = 0; i <= d; i++)
        for (int j = 0; j <= d; j++)
            g[i * (d + 1) + j] = INFINITY;
    g[0] = 0.0f;
    for (int i = 1; i <= d; i++) {
        for (int j = 1; j <= d; j++) {
            if (abs(i - j) > rho) continue;
            float diff = q[i - 1] - c[j - 1];
            float a = g[(i - 1) * (d + 1) + j], b = g[i * (d + 1) + j - 1],
                  e = g[(i - 1) * (d + 1) + j - 1];
            float m = a < b ? a : b;
            m = m < e ? m : e;
            g[i * (d + 1) + j] = fmaf(diff, diff, m);
        }
    }
    float r = g[d * (d + 1) + d];
    free(g);
    return r;
}

/* ------------------------------------------------------------------------ */
/* Suffix kNN Search, Def. 4.1, by brute force.                  */
/* For one master query MQ = mq[0..D) of a sensor series c[0..n):            */
/*   IQ_i = MQ[D-d_i .. D)        */
/*   for every t in [t_lo, min(t_hi, n-d_i+1)): D_t = DTW_{rho_i}(IQ_i, C_t) */
/*   sort (D_t, t) lexicographically (R11), keep k (multi-k by prefix,       */
/*   P:838-841), pad (R12).                                                  */
/* ------------------------------------------------------------------------ */
typedef struct { int64_t d; int64_t t; } orc_key_i64;
typedef struct { double d; int64_t t; } orc_key_f64;
typedef struct { float d; int64_t t; } orc_key_f32;

static int cmp_i64(const void *a, const void *b)
{
    const orc_key_i64 *x = a, *y = b;
    if (x->d != y->d) return x->d < y->d ? -1 : 1;
    return x->t < y->t ? -1 : (x->t > y->t);
}
static int cmp_f64(const void *a, const void *b)
{
    const orc_key_f64 *x = a, *y = b;
    if (x->d != y->d) return x->d < y->d ? -1 : 1;
    return x->t < y->t ? -1 : (x->t > y->t);
}
static int cmp_f32(const void *a, const void *b)
{
    const orc_key_f32 *x = a, *y = b;
    if (x->d != y->d) return x->d < y->d ? -1 : 1;
    return x->t < y->t ? -1 : (x->t > y->t);
}

static int64_t cand_end(int64_t n, int d, int64_t t_hi)
{
    int64_t e = n - d + 1;
    if (t_hi < e) e = t_hi;
    return e;
}

/* Returns 0, or 1 if some distance reached 2^31 (the int32 certificate of R17
 * fails; results are still exact int64). */
int orc_knn_i16(const int16_t *series, int64_t n, const int16_t *mq, int D,
                const int32_t *lengths, const int32_t *rhos, int n_len, int k,
                int64_t t_lo, int64_t t_hi, int threads,
                int64_t *ids, int64_t *dists)
{
    int over = 0;
    int64_t *c = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t *q = (int64_t *)malloc(sizeof(int64_t) * (size_t)D);
    for (int64_t i = 0; i < n; i++) c[i] = series[i];
    for (int i = 0; i < D; i++) q[i] = mq[i];
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#endif
    for (int li = 0; li < n_len; li++) {
        int d = lengths[li], rho = rhos[li];
        const int64_t *iq = q + (D - d);
        int64_t e = cand_end(n, d, t_hi);
        int64_t nc = e > t_lo ? e - t_lo : 0;
        orc_key_i64 *all = (orc_key_i64 *)malloc(sizeof(orc_key_i64) * (size_t)(nc > 0 ? nc : 1));
#pragma omp parallel for schedule(dynamic, 64) reduction(| : over)
        for (int64_t x = 0; x < nc; x++) {
            int64_t t = t_lo + x;
            all[x].d = orc_dtw_i64(iq, c + t, d, rho);
            all[x].t = t;
            if (all[x].d >= ((int64_t)1 << 31)) over |= 1;
        }
        qsort(all, (size_t)nc, sizeof(orc_key_i64), cmp_i64);
        for (int j = 0; j < k; j++) {
            ids[li * k + j] = j < nc ? all[j].t : -1;
            dists[li * k + j] = j < nc ? all[j].d : (int64_t)INT32_MAX;
        }
        free(all);
    }
    free(c);
    free(q);
    return over;
}

void orc_knn_f64(const float *series, int64_t n, const float *mq, int D,
                 const int32_t *lengths, const int32_t *rhos, int n_len, int k,
                 int64_t t_lo, int64_t t_hi, int threads,
                 int64_t *ids, double *dists)
{
    double *c = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    double *q = (double *)malloc(sizeof(double) * (size_t)D);
    for (int64_t i = 0; i < n; i++) c[i] = series[i];
    for (int i = 0; i < D; i++) q[i] = mq[i];
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#endif
    for (int li = 0; li < n_len; li++) {
        int d = lengths[li], rho = rhos[li];
        const double *iq = q + (D - d);
        int64_t e = cand_end(n, d, t_hi);
        int64_t nc = e > t_lo ? e - t_lo : 0;
        orc_key_f64 *all = (orc_key_f64 *)malloc(sizeof(orc_key_f64) * (size_t)(nc > 0 ? nc : 1));
#pragma omp parallel for schedule(dynamic, 64)
        for (int64_t x = 0; x < nc; x++) {
            int64_t t = t_lo + x;
            all[x].d = orc_dtw_f64(iq, c + t, d, rho);
            all[x].t = t;
        }
        qsort(all, (size_t)nc, sizeof(orc_key_f64), cmp_f64);
        for (int j = 0; j < k; j++) {
            ids[li * k + j] = j < nc ? all[j].t : -1;
            dists[li * k + j] = j < nc ? all[j].d : INFINITY;
        }
        free(all);
    }
    free(c);
    free(q);
}

void orc_knn_f32(const float *series, int64_t n, const float *mq, int D,
                 const int32_t *lengths, const int32_t *rhos, int n_len, int k,
                 int64_t t_lo, int64_t t_hi, int threads,
                 int64_t *ids, float *dists)
{
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#endif
    for (int li = 0; li < n_len; li++) {
        int d = lengths[li], rho = rhos[li];
        const float *iq = mq + (D - d);
        int64_t e = cand_end(n, d, t_hi);
        int64_t nc = e > t_lo ? e - t_lo : 0;
        orc_key_f32 *all = (orc_key_f32 *)malloc(sizeof(orc_key_f32) * (size_t)(nc > 0 ? nc : 1));
#pragma omp parallel for schedule(dynamic, 64)
        for (int64_t x = 0; x < nc; x++) {
            int64_t t = t_lo + x;
            all[x].d = orc_dtw_f32(iq, series + t, d, rho);
            all[x].t = t;
        }
        qsort(all, (size_t)nc, sizeof(orc_key_f32), cmp_f32);
        for (int j = 0; j < k; j++) {
            ids[li * k + j] = j < nc ? all[j].t : -1;
            dists[li * k + j] = j < nc ? all[j].d : INFINITY;
        }
        free(all);
    }
}

/* DTW of a given list of candidates (used to check any single verified value). */
void orc_dtw_list_i16(const int16_t *series, const int16_t *q16, int d, int rho,
                      const int64_t *ts, int64_t nt, int64_t *out)
{
    int64_t *q = (int64_t *)malloc(sizeof(int64_t) * (size_t)d);
    int64_t *c = (int64_t *)malloc(sizeof(int64_t) * (size_t)d);
    for (int i = 0; i < d; i++) q[i] = q16[i];
    for (int64_t x = 0; x < nt; x++) {
        for (int i = 0; i < d; i++) c[i] = series[ts[x] + i];
        out[x] = orc_dtw_i64(q, c, d, rho);
    }
    free(q);
    free(c);
}

void orc_dtw_list_f32(const float *series, const float *q, int d, int rho,
                      const int64_t *ts, int64_t nt, float *out32, double *out64)
{
    double *qd = (double *)malloc(sizeof(double) * (size_t)d);
    double *cd = (double *)malloc(sizeof(double) * (size_t)d);
    for (int i = 0; i < d; i++) qd[i] = q[i];
    for (int64_t x = 0; x < nt; x++) {
        out32[x] = orc_dtw_f32(q, series + ts[x], d, rho);
        for (int i = 0; i < d; i++) cd[i] = series[ts[x] + i];
        out64[x] = orc_dtw_f64(qd, cd, d, rho);
    }
    free(qd);
    free(cd);
}

/* ------------------------------------------------------------------------ */
/* Lower bounds.                                                             */
/*                                                                           */
/* Point term of LB_Keogh, Eq. 26 and the per-point form used  */
/* in the proof of Thm. 4.3:                                   */
/*   e(v; U, L) = dist(U, v) if v > U;  dist(L, v) if v < L;  0 otherwise.   */
/* LB_EQ(Q,C) = LB_keogh(E(Q), C),  LB_EC(Q,C) = LB_keogh(E(C), Q)*/
/* LB_en = max(LB_EQ, LB_EC)                                  (Thm 4.1) */
/* ------------------------------------------------------------------------ */
static int64_t e_i64(int64_t v, int64_t U, int64_t L)
{
    if (v > U) return (v - U) * (v - U);
    if (v < L) return (L - v) * (L - v);
    return 0;
}
static double e_f64(double v, double U, double L)
{
    if (v > U) return (v - U) * (v - U);
    if (v < L) return (L - v) * (L - v);
    return 0.0;
}

/* Window-level posting lists (Sec. 4.3.1; Fig. 4-5):
 * SW_b = MQ[D-w-b .. D-b)  for b in [0, D-w]         (R19)
 * DW_r = c[r*w .. r*w+w)   for r in [0, floor(n/w))
 * P_EQ[b][r] = LB_keogh(E(MQ) restricted to SW_b, DW_r)
 * P_EC[b][r] = LB_keogh(E(C) restricted to DW_r, SW_b)
 * The envelopes UQ/LQ (of the whole MQ, R20) and UC/LC (of the whole series)
 * are inputs, computed by orc_envelope_*.  Output layout [b][r]. */
void orc_postings_i64(const int64_t *c, int64_t n, const int64_t *UC, const int64_t *LC,
                      const int64_t *mq, const int64_t *UQ, const int64_t *LQ, int D, int w,
                      int64_t *P_EQ, int64_t *P_EC)
{
    int n_sw = D - w + 1;
    int64_t n_dw = n / w;
    for (int b = 0; b < n_sw; b++) {
        int p0 = D - w - b;
        for (int64_t r = 0; r < n_dw; r++) {
            int64_t eq = 0, ec = 0;
            for (int j = 0; j < w; j++) {
                int64_t s = r * w + j;
                int p = p0 + j;
                eq += e_i64(c[s], UQ[p], LQ[p]);
                ec += e_i64(mq[p], UC[s], LC[s]);
            }
            P_EQ[(int64_t)b * n_dw + r] = eq;
            P_EC[(int64_t)b * n_dw + r] = ec;
        }
    }
}

void orc_postings_f64(const double *c, int64_t n, const double *UC, const double *LC,
                      const double *mq, const double *UQ, const double *LQ, int D, int w,
                      double *P_EQ, double *P_EC)
{
    int n_sw = D - w + 1;
    int64_t n_dw = n / w;
    for (int b = 0; b < n_sw; b++) {
        int p0 = D - w - b;
        for (int64_t r = 0; r < n_dw; r++) {
            double eq = 0, ec = 0;
            for (int j = 0; j < w; j++) {
                int64_t s = r * w + j;
                int p = p0 + j;
                eq += e_f64(c[s], UQ[p], LQ[p]);
                ec += e_f64(mq[p], UC[s], LC[s]);
            }
            P_EQ[(int64_t)b * n_dw + r] = eq;
            P_EC[(int64_t)b * n_dw + r] = ec;
        }
    }
}

/* Per-candidate lower bounds of IQ_i = MQ[D-d .. D) against C_{t,d} for every
 * t in [0, n-d]:
 *   p(s) = s - t + (D - d)   (the MQ position aligned with series point s)
 *   LB_EQ = sum_{s=t}^{t+d-1} e(c[s]; UQ[p], LQ[p])
 *   LB_EC = sum_{s=t}^{t+d-1} e(MQ[p]; UC[s], LC[s])
 *   LB_en = max(LB_EQ, LB_EC)
 * LB_w (Thm. 4.3 / Eq. 5) restricted to the m full disjoint
 * windows inside the segment, derived here from t (not from (b, r)):
 *   r      = floor((t+d)/w) - 1        rightmost full DW
 *   r_left = ceil(t/w)                 leftmost full DW
 *   m      = r - r_left + 1
 *   b      = t + d - (r+1) w           (Thm. 4.2 proof)
 *   LB_w   = max(sum over s in [r_left w, (r+1) w) of the EQ terms,
 *                same for the EC terms)              if m >= 1, else 0 (R6)
 * Outputs (each [n-d+1]): lb_eq, lb_ec, lb_en, lb_w, and b, r, m; lb_weq and
 * lb_wec (may be NULL) are the two sums inside LB_w's max (Eq. 5), the bounds
 * of Table 3's "LB_EQ" / "LB_EC" rows over the full windows. */
void orc_lb_i64(const int64_t *c, int64_t n, const int64_t *UC, const int64_t *LC,
                const int64_t *mq, const int64_t *UQ, const int64_t *LQ, int D, int d, int w,
                int64_t *lb_eq, int64_t *lb_ec, int64_t *lb_en, int64_t *lb_w,
                int64_t *ob, int64_t *orr, int64_t *om, int64_t *lb_weq, int64_t *lb_wec)
{
    for (int64_t t = 0; t + d <= n; t++) {
        int64_t eq = 0, ec = 0, weq = 0, wec = 0;
        int64_t r = (t + d) / w - 1;
        int64_t r_left = (t + w - 1) / w;
        int64_t m = r - r_left + 1;
        for (int64_t s = t; s < t + d; s++) {
            int64_t p = s - t + (D - d);
            int64_t te = e_i64(c[s], UQ[p], LQ[p]);
            int64_t tc = e_i64(mq[p], UC[s], LC[s]);
            eq += te;
            ec += tc;
            if (m >= 1 && s >= r_left * w && s < (r + 1) * w) {
                weq += te;
                wec += tc;
            }
        }
        lb_eq[t] = eq;
        lb_ec[t] = ec;
        lb_en[t] = eq > ec ? eq : ec;
        lb_w[t] = m >= 1 ? (weq > wec ? weq : wec) : 0;
        if (lb_weq) lb_weq[t] = m >= 1 ? weq : 0;
        if (lb_wec) lb_wec[t] = m >= 1 ? wec : 0;
        ob[t] = t + d - (r + 1) * w;
        orr[t] = r;
        om[t] = m;
    }
}

void orc_lb_f64(const double *c, int64_t n, const double *UC, const double *LC,
                const double *mq, const double *UQ, const double *LQ, int D, int d, int w,
                double *lb_eq, double *lb_ec, double *lb_en, double *lb_w, double *lb_weq, double *lb_wec)
{
    for (int64_t t = 0; t + d <= n; t++) {
        double eq = 0, ec = 0, weq = 0, wec = 0;
        int64_t r = (t + d) / w - 1;
        int64_t r_left = (t + w - 1) / w;
        int64_t m = r - r_left + 1;
        for (int64_t s = t; s < t + d; s++) {
            int64_t p = s - t + (D - d);
            double te = e_f64(c[s], UQ[p], LQ[p]);
            double tc = e_f64(mq[p], UC[s], LC[s]);
            eq += te;
            ec += tc;
            if (m >= 1 && s >= r_left * w && s < (r + 1) * w) {
                weq += te;
                wec += tc;
            }
        }
        lb_eq[t] = eq;
        lb_ec[t] = ec;
        lb_en[t] = eq > ec ? eq : ec;
        lb_w[t] = m >= 1 ? (weq > wec ? weq : wec) : 0.0;
        if (lb_weq) lb_weq[t] = m >= 1 ? weq : 0.0;
        if (lb_wec) lb_wec[t] = m >= 1 ? wec : 0.0;
    }
}
