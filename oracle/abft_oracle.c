/*
 * oracle/abft_oracle.c — CPU ORACLE, TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct FP64 implementation of the Enhanced Online-ABFT blocked
 * Cholesky of Chen, Liang & Chen (PAPER.md, IPDPS'16), written from the paper. Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load it. It shares no code, header, table or constant with the CUDA path under
 * paper_conf_ipps_chenlc16_b200/ and never calls it.
 *
 * Paper anchors (PAPER.md line, section):
 *   encode            chk1 = v1^T A, chk2 = v2^T A, v1=[1..1], v2=[1..B]     121-129  §IV.A
 *   SYRK/GEMM update  A' = A - LC LC^T ; chk(A') = chk(A) - chk(LC) LC^T      137-153  §IV.B
 *   POTF2 + Alg. 2    chk[j] /= LA[j,j]; chk[j+1:] -= chk[j] LA[j+1:, j]      155-168  §IV.B
 *   TRSM              LB = B' (LA^T)^-1 ; chk(LB) = chk(B') (LA^T)^-1         170-176  §IV.B
 *   detect/locate     d1 = r1' - r1, d2 = r2' - r2, |d1| > e, d2/d1 = j      180-195  §IV.C
 *   verify-before-use ("data blocks are verified before each time they are referenced")
 *                                                                            100-107  §III
 *   verify every K iterations (Opt. 3)                                       253-267  §V.C
 * Readings where the paper is silent or garbled are SURVEY.md §8c A1..A22 / DESIGN.md §3;
 * the ones used here are cited inline as [Ann].
 *
 * Loop order is right-looking [A1]. All arithmetic is IEEE FP64, compiled with
 * -ffp-contract=off and no -ffast-math. Parallelism is plain OpenMP over independent tiles /
 * columns; within one sum the order is ascending index, so results do not depend on the
 * thread count.
 *
 * Parity status of each function is recorded in DESIGN.md §4 ("pins"). The threshold
 * constants C_tau and rho [A4, A6] are "parity unpinned" by the paper; they are pinned only
 * by the noise measurements the test-suite re-runs (tests/test_oracle_pins.py::test_noise_margin).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---- codes (restated from the interface contract, not included from include/) ---------- */
enum { O_HOOK_REST = 0, O_HOOK_POTRF_OUT = 1, O_HOOK_TRSM_OUT = 2, O_HOOK_UPDATE_OUT = 3, O_HOOK_RECV = 4 };
enum { O_TGT_DATA = 0, O_TGT_CHK = 1 };
enum { O_V1 = 1, O_V2 = 2, O_V3 = 3, O_V4 = 4, O_V5 = 5, O_V6 = 6, O_V4R = 7, O_V7 = 8 };
enum { O_DATA = 1, O_NONFINITE = 2, O_CHK1 = 3, O_CHK2 = 4, O_UNCORRECTABLE = 5, O_CHK3 = 6 };
enum { O_OK = 0, O_STATUS_UNCORRECTABLE = 1, O_STATUS_NOT_SPD = 2 };

typedef struct { int32_t k, hook, target, pad0; int64_t row, col; uint64_t xor_mask; int32_t rank, pad1; } oinj_t;
typedef struct { int32_t k, check, tile_i, tile_j, row, col, kind, rank; double delta1, delta2; } oevent_t;
typedef struct {
    int64_t n_checks, n_detected, n_data, n_nonfinite, n_chk1, n_chk2, n_uncorrectable;
    double flops_factor;     /* POTRF + TRSM + update on data rows                          */
    double flops_chkupd;     /* Alg. 2 + TRSM on checksum rows + update of checksum rows     */
    double flops_check;      /* checksum recalculation (4 flops per element: P:285 convention)*/
    double flops_encode;
    double bytes_check;      /* 8 bytes per element read by a check                          */
    double max_ratio;        /* max over passing columns of max(|d1|/tau1, |d2|/tau2): noise */
} ocount_t;

#define EPS 0x1p-52          /* DBL_EPSILON [A17] */

typedef struct {
    int64_t n, B, N, lda, ldc;
    int nchk;                      /* checksum rows per block: 2 (the paper's choice) or 3
                                      (m+1 = 3 for m = 2 errors per column; NEXT-4)      */
    double *A, *chk, *s, *S1, *S2, *S3;
    double c_tau, rho;
    int nranks, K, correct;
    int prows;                     /* P>1 simulation: process grid prows x (nranks / prows); tile (I,J)
                                      belongs to rank (I mod prows) * pcols + (J mod pcols) — 2D
                                      block-cyclic; prows = 1 is the 1D column cyclic */
    int mode;                      /* 0 Enhanced Online-ABFT, 1 Online-ABFT, 2 Offline-ABFT */
    const oinj_t* inj; int64_t ninj;
    oevent_t* ev; int64_t cap, nev;
    int status; int64_t info;
    ocount_t* cnt;
} octx_t;

/* A tile "view": data pointer + leading dim, two checksum rows (pointer + stride). */
typedef struct {
    double* T; int64_t ldt;
    double* c1; double* c2; int64_t ldc;   /* chk1[c] = c1[c*ldc], chk2[c] = c2[c*ldc] */
    double* c3;                            /* third checksum row (v3 = [1, 4, ..., B^2]) or NULL */
    int64_t I, J;                          /* tile coordinates (for scales / events)    */
    int diag, factored;
} tview_t;

/* The logical tile X of the check [A12]: sym(tril(T)) for an unfactored diagonal tile,
 * tril(T) for a factored one, T otherwise. */
static inline double X(const tview_t* v, int64_t r, int64_t c) {
    if (v->diag) {
        if (r >= c) return v->T[c * v->ldt + r];
        return v->factored ? 0.0 : v->T[r * v->ldt + c];
    }
    return v->T[c * v->ldt + r];
}
/* the stored element behind X(r,c) */
static inline double* Xstore(const tview_t* v, int64_t r, int64_t c) {
    if (v->diag && r < c) return &v->T[r * v->ldt + c];
    return &v->T[c * v->ldt + r];
}

static void push_event(octx_t* x, int k, int V, const tview_t* v, int64_t row, int64_t col, int kind,
                       int rank, double d1, double d2) {
    if (x->nev < x->cap && x->ev) {
        oevent_t* e = &x->ev[x->nev];
        e->k = k; e->check = V; e->tile_i = (int32_t)v->I; e->tile_j = (int32_t)v->J;
        e->row = (int32_t)row; e->col = (int32_t)col; e->kind = kind; e->rank = rank;
        e->delta1 = d1; e->delta2 = d2;
    }
    x->nev++;
}

/* ---- Check(T(I,J)) — PAPER.md:180-195 §IV.C with readings A4-A12 ---------------------- */
typedef struct { int64_t c; int kind; int64_t row, row2; double d1, d2, d3, r1, r2, r3; } odec_t;

/* Two errors in one column from three weighted sums (NEXT-4; "m+1 column checksums could
 * locate and correct up to m errors per column", reading B10). With errors Da at weight wa and Db
 * at weight wb (weights 1..B): d1 = Da + Db, d2 = wa Da + wb Db, d3 = wa^2 Da + wb^2 Db, so
 * d3 = S d2 - P d1 with S = wa + wb, P = wa wb. Scan S = 3 .. 2B-1 in ascending order, P = rint((S d2 -
 * d3) / d1); accept (wa, wb) = (S -+ sqrt(S^2 - 4P)) / 2 if they are integers in 1..B, the residual
 * d3 - S d2 + P d1 is within its rounding tolerance and both errors exceed tau1. Exactly one
 * accepted pair locates the errors; none or several -> not located. Returns 1 and the 0-based rows. */
#define RHO2 0x1p-40   /* relative slack of the two-error residual [B10]: the single-error 2^-30 [A6]
                         would let a large error's slack hide a small second error (ambiguity);
                         2^-40 still exceeds the worst-case relative rounding of the sums, B eps */
static int locate_two(double d1, double d2, double d3, double tau1, double tau2, double tau3, double rho, int64_t B,
                      int64_t* ra, int64_t* rb) {
    (void)rho;
    rho = RHO2;
    int found = 0;
    if (!(fabs(d1) > tau1)) return 0;                 /* Da + Db ~ 0: P is not determined */
    for (int64_t S = 3; S <= 2 * B - 1; ++S) {
        const double Sd = (double)S;
        const double Pd = nearbyint((Sd * d2 - d3) / d1);
        if (!(Pd >= 2.0) || Pd > (double)B * (double)(B - 1)) continue;
        const int64_t P = (int64_t)Pd;
        const int64_t disc = S * S - 4 * P;
        if (disc <= 0) continue;
        int64_t q = (int64_t)sqrt((double)disc);
        while (q * q > disc) --q;
        while ((q + 1) * (q + 1) <= disc) ++q;
        if (q * q != disc || ((S - q) & 1)) continue;
        const int64_t wa = (S - q) / 2, wb = (S + q) / 2;
        if (wa < 1 || wb > B) continue;
        const double res = d3 - Sd * d2 + Pd * d1;
        /* the thresholds bound each sum's fault-free noise with a wide margin (P9: measured <= 2^-6
         * of tau); their full combination admits false pairs, so the residual allows 1/16 of it */
        const double tol = (tau3 + Sd * tau2 + Pd * tau1) * 0.0625 + rho * (fabs(d3) + Sd * fabs(d2) + Pd * fabs(d1));
        if (!(fabs(res) <= tol)) continue;
        const double Da = ((double)wb * d1 - d2) / (double)(wb - wa), Db = (d2 - (double)wa * d1) / (double)(wb - wa);
        if (!(fabs(Da) > tau1) || !(fabs(Db) > tau1)) continue;
        if (++found == 1) { *ra = wa - 1; *rb = wb - 1; }
    }
    return found == 1;
}

/* the rank that owns (stores, updates and checks) tile (I, J) of the P>1 simulation */
static int tile_owner(const octx_t* x, int64_t I, int64_t J) {
    const int pr = x->prows > 0 ? x->prows : 1, pc = x->nranks / pr;
    return (int)((I % pr) * pc + (J % pc));
}

static int check_tile(octx_t* x, const tview_t* v, int k, int V, int rank) {
    const int64_t B = x->B;
    if (V != O_V4R) rank = tile_owner(x, v->I, v->J);   /* the owner of tile (I, J) runs the check */
    odec_t* dec = (odec_t*)malloc(sizeof(odec_t) * (size_t)B);
    int64_t nd = 0;
    x->cnt->n_checks++;
    x->cnt->flops_check += 2.0 * x->nchk * (double)(B * B);
    x->cnt->bytes_check += 8.0 * (double)(v->diag ? B * (B + 1) / 2 : B * B);
    for (int64_t c = 0; c < B; ++c) {
        /* recalculation chk' = v^T X, ascending row order */
        double r1 = 0.0, r2 = 0.0, r3 = 0.0;
        for (int64_t r = 0; r < B; ++r) {
            double xv = X(v, r, c);
            r1 += xv;
            r2 += (double)(r + 1) * xv;          /* v2 = [1, 2, ..., B] [A7] */
            if (v->c3) r3 += (double)((r + 1) * (r + 1)) * xv;   /* v3 = [1, 4, ..., B^2] [B10] */
        }
        const double chk1 = v->c1[c * v->ldc], chk2 = v->c2[c * v->ldc];
        const double d1 = r1 - chk1, d2 = r2 - chk2;
        const double d3 = v->c3 ? r3 - v->c3[c * v->ldc] : 0.0;
        const int64_t g = v->J * B + c;
        const double sc = v->factored ? 1.0 : x->s[g];
        const double tau1 = ((x->c_tau * EPS) * x->S1[v->I]) * sc;   /* [A4] */
        const double tau2 = ((x->c_tau * EPS) * x->S2[v->I]) * sc;
        const double tau3 = v->c3 ? ((x->c_tau * EPS) * x->S3[v->I]) * sc : 0.0;
        const int f1 = !isfinite(d1) || fabs(d1) > tau1;             /* P:195 + [A5] */
        const int f2 = !isfinite(d2) || fabs(d2) > tau2;
        const int f3 = v->c3 ? (!isfinite(d3) || fabs(d3) > tau3) : 0;
        if (!f1 && !f2 && !f3) {
            const double q1 = fabs(d1) / tau1, q2 = fabs(d2) / tau2;
            if (q1 > x->cnt->max_ratio) x->cnt->max_ratio = q1;
            if (q2 > x->cnt->max_ratio) x->cnt->max_ratio = q2;
            if (v->c3 && fabs(d3) / tau3 > x->cnt->max_ratio) x->cnt->max_ratio = fabs(d3) / tau3;
            continue;
        }
        odec_t* dd = &dec[nd++];
        dd->c = c; dd->d1 = d1; dd->d2 = d2; dd->d3 = d3; dd->r1 = r1; dd->r2 = r2; dd->r3 = r3;
        dd->row = -1; dd->row2 = -1;
        if (!isfinite(d1) || !isfinite(d2) || !isfinite(d3)) {       /* [A9] */
            int64_t best = 0; double bv = -1.0;
            for (int64_t r = 0; r < B; ++r) {
                double xv = X(v, r, c);
                double m = isfinite(xv) ? fabs(xv) : INFINITY;
                if (m > bv) { bv = m; best = r; }
            }
            dd->kind = O_NONFINITE; dd->row = best;
            continue;
        }
        if (f1) {                                                    /* locate: j = d2/d1 [A6] */
            const double q = d2 / d1;
            const double j = nearbyint(q);                           /* round half to even */
            if (j >= 1.0 && j <= (double)B) {
                const double jd1 = j * d1;
                const double j2d1 = (j * j) * d1;
                if (fabs(d2 - jd1) <= tau2 + x->rho * fabs(jd1) &&
                    (!v->c3 || fabs(d3 - j2d1) <= tau3 + x->rho * fabs(j2d1))) {
                    dd->kind = O_DATA; dd->row = (int64_t)j - 1;     /* 1-based weights [A7] */
                    continue;
                }
            }
        }
        if (f1 + f2 + f3 == 1) {                                     /* one checksum row corrupted [A10] */
            dd->kind = f1 ? O_CHK1 : f2 ? O_CHK2 : O_CHK3;
            continue;
        }
        if (v->c3 && locate_two(d1, d2, d3, tau1, tau2, tau3, x->rho, B, &dd->row, &dd->row2)) {
            dd->kind = O_DATA;                                       /* two data errors [B10] */
            continue;
        }
        dd->kind = O_UNCORRECTABLE;
    }
    /* corrections, computed from the pre-correction X, then applied [A8, A12] */
    typedef struct { double* p; double val; } fix_t;
    fix_t* fix = (fix_t*)malloc(sizeof(fix_t) * (size_t)(2 * nd + 1));
    int64_t nf = 0; int unc = 0;
    for (int64_t t = 0; t < nd; ++t) {
        odec_t* dd = &dec[t];
        const int64_t c = dd->c;
        x->cnt->n_detected++;
        if ((dd->kind == O_DATA && dd->row2 < 0) || dd->kind == O_NONFINITE) {
            double* p = Xstore(v, dd->row, c);
            int dup = 0;
            for (int64_t u = 0; u < nf; ++u) if (fix[u].p == p) dup = 1;
            if (dup) { x->cnt->n_detected--; continue; }   /* dedupe: corrected once, logged once */
            double sum = 0.0;                              /* chk1[c] - sum_{r != row} X[r,c] [A8] */
            for (int64_t r = 0; r < B; ++r) if (r != dd->row) sum += X(v, r, c);
            fix[nf].p = p; fix[nf].val = v->c1[c * v->ldc] - sum; nf++;
            int64_t sr = dd->row, scn = c;
            if (v->diag && !v->factored && sr < scn) { int64_t t2 = sr; sr = scn; scn = t2; }
            push_event(x, k, V, v, sr, scn, dd->kind, rank, dd->d1, dd->d2);
            if (dd->kind == O_DATA) x->cnt->n_data++; else x->cnt->n_nonfinite++;
        } else if (dd->kind == O_DATA) {                   /* two errors: rows a < b [B10] */
            const int64_t ra = dd->row, rb = dd->row2;
            const double wa = (double)(ra + 1), wb = (double)(rb + 1);
            double s1 = 0.0, s2 = 0.0;                     /* the other B-2 rows, summed directly [A8] */
            for (int64_t r = 0; r < B; ++r) {
                if (r == ra || r == rb) continue;
                const double xv = X(v, r, c);
                s1 += xv; s2 += (double)(r + 1) * xv;
            }
            const double R1 = v->c1[c * v->ldc] - s1, R2 = v->c2[c * v->ldc] - s2;
            const double xa = (wb * R1 - R2) / (wb - wa), xb = (R2 - wa * R1) / (wb - wa);
            const int64_t rows[2] = {ra, rb};
            const double vals[2] = {xa, xb};
            int logged = 0;
            for (int h = 0; h < 2; ++h) {
                double* p = Xstore(v, rows[h], c);
                int dup = 0;
                for (int64_t u = 0; u < nf; ++u) if (fix[u].p == p) dup = 1;
                if (dup) continue;
                fix[nf].p = p; fix[nf].val = vals[h]; nf++;
                int64_t sr = rows[h], scn = c;
                if (v->diag && !v->factored && sr < scn) { int64_t t2 = sr; sr = scn; scn = t2; }
                push_event(x, k, V, v, sr, scn, O_DATA, rank, dd->d1, dd->d2);
                x->cnt->n_data++;
                logged++;
            }
            x->cnt->n_detected += logged - 1;
        } else if (dd->kind == O_CHK1) {
            push_event(x, k, V, v, -1, c, O_CHK1, rank, dd->d1, dd->d2);
            x->cnt->n_chk1++;
        } else if (dd->kind == O_CHK2) {
            push_event(x, k, V, v, -2, c, O_CHK2, rank, dd->d1, dd->d2);
            x->cnt->n_chk2++;
        } else if (dd->kind == O_CHK3) {
            push_event(x, k, V, v, -4, c, O_CHK3, rank, dd->d1, dd->d2);
            x->cnt->n_chk2++;
        } else {
            push_event(x, k, V, v, -3, c, O_UNCORRECTABLE, rank, dd->d1, dd->d2);
            x->cnt->n_uncorrectable++;
            unc = 1;
        }
    }
    if (x->correct) {
        for (int64_t u = 0; u < nf; ++u) *fix[u].p = fix[u].val;
        for (int64_t t = 0; t < nd; ++t) {
            if (dec[t].kind == O_CHK1) v->c1[dec[t].c * v->ldc] = dec[t].r1;   /* chk1 := v1^T X */
            if (dec[t].kind == O_CHK2) v->c2[dec[t].c * v->ldc] = dec[t].r2;   /* chk2 := v2^T X */
            if (dec[t].kind == O_CHK3) v->c3[dec[t].c * v->ldc] = dec[t].r3;   /* chk3 := v3^T X */
        }
    }
    free(fix); free(dec);
    if (unc) x->status = O_STATUS_UNCORRECTABLE;
    return unc;
}

/* ---- views into the global matrix ------------------------------------------------------ */
static tview_t gview(octx_t* x, int64_t I, int64_t J, int factored) {
    tview_t v;
    v.T = x->A + J * x->B * x->lda + I * x->B; v.ldt = x->lda;
    v.c1 = x->chk + J * x->B * x->ldc + x->nchk * I; v.c2 = v.c1 + 1; v.ldc = x->ldc;
    v.c3 = x->nchk == 3 ? v.c1 + 2 : NULL;
    v.I = I; v.J = J; v.diag = (I == J); v.factored = factored;
    return v;
}

/* ---- encoding: §IV.A, P:285 -------------------------------------------- */
static void scales(octx_t* x) {
    const int64_t n = x->n, B = x->B;
    for (int64_t i = 0; i < n; ++i) x->s[i] = sqrt(x->A[i * x->lda + i]);    /* s_i = sqrt(A_ii) [A4] */
    for (int64_t I = 0; I < x->N; ++I) {
        double a = 0.0, b = 0.0, c = 0.0;
        for (int64_t r = 0; r < B; ++r) {
            a += x->s[I * B + r]; b += (double)(r + 1) * x->s[I * B + r];
            c += (double)((r + 1) * (r + 1)) * x->s[I * B + r];   /* S3 for v3 [B10] */
        }
        x->S1[I] = a; x->S2[I] = b;
        if (x->S3) x->S3[I] = c;
    }
}

static void encode(octx_t* x) {
    const int64_t B = x->B, N = x->N;
    #pragma omp parallel for schedule(dynamic)
    for (int64_t g = 0; g < N * B; ++g) {             /* global column g, all tiles I >= J */
        const int64_t J = g / B, c = g % B;
        for (int64_t I = J; I < N; ++I) {
            tview_t v = gview(x, I, J, 0);
            double r1 = 0.0, r2 = 0.0, r3 = 0.0;
            for (int64_t r = 0; r < B; ++r) {
                double xv = X(&v, r, c); r1 += xv; r2 += (double)(r + 1) * xv;
                r3 += (double)((r + 1) * (r + 1)) * xv;
            }
            v.c1[c * v.ldc] = r1; v.c2[c * v.ldc] = r2;
            if (v.c3) v.c3[c * v.ldc] = r3;
        }
    }
    x->cnt->flops_encode += 2.0 * x->nchk * (double)(N * (N + 1) / 2) * (double)(B * B);
}

/* ---- fault injection at a named hook [A16, A21] ----------------------------------------- */
static void xor_double(double* p, uint64_t m) { uint64_t u; memcpy(&u, p, 8); u ^= m; memcpy(p, &u, 8); }

static void inject(octx_t* x, int k, int hook, int rank, double* A, int64_t lda, double* chk, int64_t ldc) {
    for (int64_t t = 0; t < x->ninj; ++t) {
        const oinj_t* s = &x->inj[t];
        if (s->k != k || s->hook != hook) continue;
        if (hook == O_HOOK_RECV && s->rank != rank) continue;
        if (s->target == O_TGT_DATA) xor_double(&A[s->col * lda + s->row], s->xor_mask);
        else xor_double(&chk[s->col * ldc + s->row], s->xor_mask);
    }
}

/* ---- POTF2 on sym(T(k,k)) + Alg. 2 ---------------------------------- */
static int potrf_tile(octx_t* x, int64_t k) {
    const int64_t B = x->B, lda = x->lda;
    double* T = x->A + k * B * lda + k * B;
    for (int64_t j = 0; j < B; ++j) {                 /* unblocked Cholesky (dpotf2 order) */
        double ajj = T[j * lda + j];
        for (int64_t p = 0; p < j; ++p) ajj -= T[p * lda + j] * T[p * lda + j];
        if (!(ajj > 0.0)) { x->status = O_STATUS_NOT_SPD; x->info = k * B + j + 1; return 1; }
        const double ljj = sqrt(ajj);
        T[j * lda + j] = ljj;
        for (int64_t i = j + 1; i < B; ++i) {
            double a = T[j * lda + i];
            for (int64_t p = 0; p < j; ++p) a -= T[p * lda + i] * T[p * lda + j];
            T[j * lda + i] = a / ljj;
        }
    }
    x->cnt->flops_factor += (double)B * B * B / 3.0;
    /* Alg. 2, on both checksum rows of tile (k,k) [A3] */
    for (int t = 0; t < x->nchk; ++t) {
        double* ck = x->chk + k * B * x->ldc + x->nchk * k + t;
        const int64_t st = x->ldc;
        for (int64_t j = 0; j < B; ++j) {
            ck[j * st] = ck[j * st] / T[j * lda + j];                         /* line 2 */
            for (int64_t i = j + 1; i < B; ++i) ck[i * st] -= ck[j * st] * T[j * lda + i];   /* line 3 */
        }
    }
    x->cnt->flops_chkupd += (double)x->nchk * B * B;
    return 0;
}

/* ---- TRSM: row-wise forward substitution x L^T = b ------------------ */
static void trsm_row(const double* L, int64_t lda, int64_t B, double* b, int64_t stride) {
    for (int64_t j = 0; j < B; ++j) {
        b[j * stride] = b[j * stride] / L[j * lda + j];
        for (int64_t i = j + 1; i < B; ++i) b[i * stride] -= b[j * stride] * L[j * lda + i];
    }
}

static void trsm_panel(octx_t* x, int64_t k) {
    const int64_t B = x->B, N = x->N, lda = x->lda, n = x->n;
    const double* L = x->A + k * B * lda + k * B;
    /* Data rows: the same per-element operation sequence as trsm_row (b[j] /= L[j,j], then
     * b[i] -= b[j] L[i,j] for i > j, j ascending), with rows as the inner loop so that the
     * column-major panel is walked contiguously. Row blocks are independent. */
    const int64_t r0 = (k + 1) * B, RB = 64;
    #pragma omp parallel for schedule(static)
    for (int64_t rb = r0; rb < n; rb += RB) {
        const int64_t re = rb + RB < n ? rb + RB : n;
        double* P = x->A + k * B * lda;
        for (int64_t j = 0; j < B; ++j) {
            const double d = L[j * lda + j];
            for (int64_t r = rb; r < re; ++r) P[j * lda + r] = P[j * lda + r] / d;
            for (int64_t i = j + 1; i < B; ++i) {
                const double l = L[j * lda + i];
                for (int64_t r = rb; r < re; ++r) P[i * lda + r] -= P[j * lda + r] * l;
            }
        }
    }
    for (int64_t r = x->nchk * (k + 1); r < x->nchk * N; ++r) trsm_row(L, lda, B, x->chk + k * B * x->ldc + r, x->ldc);
    x->cnt->flops_factor += (double)(n - (k + 1) * B) * B * B;
    x->cnt->flops_chkupd += (double)(x->nchk * (N - k - 1)) * B * B;
}

/* ---- trailing update: T(i,j) -= L_ik L_jk^T, chk(i,j) -= chk(i,k) L_jk^T ---
 * pan_of_rank[r] is the panel copy rank r holds (P>1 simulation); tile (i, j) is updated by its
 * owner with that rank's copy. At P=1 every copy is the panel stored in A / chk. */
typedef struct { const double* L; int64_t ldl; const double* C; int64_t ldcc; } panel_t;

static void update(octx_t* x, int64_t k, const panel_t* pan_of_rank) {
    const int64_t B = x->B, N = x->N;
    const int64_t m = N - k - 1;
    const int64_t npairs = m * (m + 1) / 2;
    #pragma omp parallel
    {
        double* tmp = (double*)malloc(sizeof(double) * (size_t)B);
        #pragma omp for schedule(dynamic)
        for (int64_t q = 0; q < npairs; ++q) {
            /* q -> (j, i) with k < j <= i < N, column-major tile order */
            int64_t jj = 0, rem = q;
            while (rem >= m - jj) { rem -= m - jj; jj++; }
            const int64_t j = k + 1 + jj, i = j + rem;
            const panel_t* P = &pan_of_rank[tile_owner(x, i, j)];   /* that rank's panel copy */
            const double* Lik = P->L + (i - k - 1) * B;      /* rows of L_ik inside the panel */
            const double* Ljk = P->L + (j - k - 1) * B;
            double* T = x->A + j * B * x->lda + i * B;
            for (int64_t c = 0; c < B; ++c) {
                const int64_t r0 = (i == j) ? c : 0;           /* lower half of diagonal tiles */
                for (int64_t r = r0; r < B; ++r) tmp[r] = 0.0;
                for (int64_t p = 0; p < B; ++p) {
                    const double l = Ljk[p * P->ldl + c];
                    for (int64_t r = r0; r < B; ++r) tmp[r] += Lik[p * P->ldl + r] * l;
                }
                for (int64_t r = r0; r < B; ++r) T[c * x->lda + r] -= tmp[r];
            }
            for (int t = 0; t < x->nchk; ++t) {               /* checksum rows */
                const double* ck = P->C + x->nchk * (i - k - 1) + t;  /* chk(i,k) row */
                double* cd = x->chk + j * B * x->ldc + x->nchk * i + t;
                for (int64_t c = 0; c < B; ++c) {
                    double a = 0.0;
                    for (int64_t p = 0; p < B; ++p) a += ck[p * P->ldcc] * Ljk[p * P->ldl + c];
                    cd[c * x->ldc] -= a;
                }
            }
        }
        free(tmp);
    }
    const double mB = (double)(m * B);
    x->cnt->flops_factor += mB * mB * B;               /* ~ (m B)^2 B: SYRK+GEMM, lower half */
    x->cnt->flops_chkupd += 2.0 * x->nchk * (double)(m * (m + 1) / 2) * B * B;
}

/* ---- the factor loop --------------------------------------------- */
static int run_checks_column(octx_t* x, int64_t k, int factored, int V_diag, int V_off, int with_diag) {
    if (with_diag) { tview_t v = gview(x, k, k, factored); if (check_tile(x, &v, (int)k, V_diag, 0)) return 1; }
    for (int64_t i = k + 1; i < x->N; ++i) {
        tview_t v = gview(x, i, k, factored);
        if (check_tile(x, &v, (int)k, V_off, 0)) return 1;
    }
    return 0;
}

/* One factorisation. Which checks run depends on the scheme (§II.B, §III):
 *   mode 0 Enhanced Online-ABFT: V1..V6 (verify before every read)
 *   mode 1 Online-ABFT: verify each operation's result after it: V3, V4, V5, + final V6
 *   mode 2 Offline-ABFT: checksums carried, verified once at the end: V6 only        */
/* kstop (timing only, bench.py's bounded CPU baseline): run iterations 0..kstop-1 and stop
 * there (no V6); kstop >= N is the whole factorisation. The arithmetic is unchanged. */
static int64_t g_kstop = INT64_MAX;

static int potrf_core(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                      int nranks, int K, double c_tau, int abft, int mode, oevent_t* ev, int64_t cap,
                      int64_t* nev, int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out, int nchk,
                      int prows) {
    octx_t X_; octx_t* x = &X_;
    memset(x, 0, sizeof *x);
    x->cnt = cnt;
    x->mode = mode;
    x->nchk = nchk;
    x->n = n; x->B = nb; x->N = n / nb; x->lda = lda; x->ldc = nchk * x->N > 0 ? nchk * x->N : 1;
    x->A = A; x->c_tau = c_tau > 0 ? c_tau : 64.0; x->rho = 0x1p-30;   /* [A4, A6] */
    x->nranks = nranks; x->prows = prows; x->K = K; x->correct = 1;
    x->inj = inj; x->ninj = ninj; x->ev = ev; x->cap = cap;
    if (info) *info = 0;
    if (n == 0) { if (nev) *nev = 0; return 0; }
    const int64_t N = x->N, B = nb;
    x->chk = (double*)calloc((size_t)(x->ldc * n), sizeof(double));
    x->s = (double*)malloc(sizeof(double) * (size_t)n);
    x->S1 = (double*)malloc(sizeof(double) * (size_t)N);
    x->S2 = (double*)malloc(sizeof(double) * (size_t)N);
    x->S3 = nchk == 3 ? (double*)malloc(sizeof(double) * (size_t)N) : NULL;
    const int nc = nchk;
    /* receiver copies of the panel (P>1 simulation) */
    double* rcopy = nranks > 1 ? (double*)malloc(sizeof(double) * (size_t)(nranks * n * B)) : NULL;
    double* rchk = nranks > 1 ? (double*)malloc(sizeof(double) * (size_t)(nranks * nc * N * B)) : NULL;
    panel_t* pan = (panel_t*)malloc(sizeof(panel_t) * (size_t)nranks);

    if (abft) { scales(x); encode(x); }
    for (int64_t k = 0; k < N && k < g_kstop && x->status == O_OK; ++k) {
        if (abft) {
            inject(x, (int)k, O_HOOK_REST, 0, x->A, lda, x->chk, x->ldc);
            if (mode == 0 && run_checks_column(x, k, 0, O_V1, O_V2, 1)) break;   /* V1, V2 */
        }
        if (potrf_tile(x, k)) break;
        if (abft) {
            inject(x, (int)k, O_HOOK_POTRF_OUT, 0, x->A, lda, x->chk, x->ldc);
            tview_t v = gview(x, k, k, 1);
            if (mode != 2 && check_tile(x, &v, (int)k, O_V3, 0)) break;      /* V3 */
        }
        trsm_panel(x, k);
        if (abft) {
            inject(x, (int)k, O_HOOK_TRSM_OUT, 0, x->A, lda, x->chk, x->ldc);
            if (mode != 2 && run_checks_column(x, k, 1, 0, O_V4, 0)) break;   /* V4 */
        }
        const int64_t m = N - k - 1;
        for (int r = 0; r < nranks; ++r) {
            pan[r].L = x->A + k * B * lda + (k + 1) * B; pan[r].ldl = lda;
            pan[r].C = x->chk + k * B * x->ldc + nc * (k + 1); pan[r].ldcc = x->ldc;
        }
        if (abft && mode == 0 && nranks > 1 && m > 0) {                     /* RECV + V4R */
            /* every rank receives the panel tiles (i, k), i > k, that it does not own (their
             * owners solved them; at prows = 1 that is the whole panel from the owner of column
             * k), applies its RECV hook to its copy and re-checks the tiles it received */
            int stop = 0;
            for (int r = 0; r < nranks && !stop; ++r) {
                int received = 0;
                for (int64_t i = k + 1; i < N; ++i) received |= (tile_owner(x, i, k) != r);
                if (!received) continue;
                double* Lr = rcopy + (size_t)r * n * B;     /* receiver buffer: m*B x B, ld = m*B */
                double* Cr = rchk + (size_t)r * nc * N * B;  /* nc m x B, ld = nc m               */
                const int64_t ldl = m * B, ldr = nc * m;
                for (int64_t c = 0; c < B; ++c) {
                    memcpy(Lr + c * ldl, x->A + (k * B + c) * lda + (k + 1) * B, sizeof(double) * (size_t)(m * B));
                    for (int64_t q = 0; q < nc * m; ++q) Cr[c * ldr + q] = x->chk[(k * B + c) * x->ldc + nc * (k + 1) + q];
                }
                /* RECV(k, r): target (row, col) global -> receiver buffer coordinates; a target in a
                 * tile rank r owns is not received by it (no effect) */
                for (int64_t t = 0; t < ninj; ++t) {
                    const oinj_t* s = &inj[t];
                    if (s->k != k || s->hook != O_HOOK_RECV || s->rank != r) continue;
                    const int64_t ti = s->target == O_TGT_DATA ? s->row / B : s->row / nc;
                    if (tile_owner(x, ti, k) == r) continue;
                    if (s->target == O_TGT_DATA) xor_double(&Lr[(s->col - k * B) * ldl + (s->row - (k + 1) * B)], s->xor_mask);
                    else xor_double(&Cr[(s->col - k * B) * ldr + (s->row - nc * (k + 1))], s->xor_mask);
                }
                for (int64_t i = k + 1; i < N && !stop; ++i) {
                    if (tile_owner(x, i, k) == r) continue;
                    tview_t v;
                    v.T = Lr + (i - k - 1) * B; v.ldt = ldl;
                    v.c1 = Cr + nc * (i - k - 1); v.c2 = v.c1 + 1; v.ldc = ldr;
                    v.c3 = nc == 3 ? v.c1 + 2 : NULL;
                    v.I = i; v.J = k; v.diag = 0; v.factored = 1;
                    if (check_tile(x, &v, (int)k, O_V4R, r)) stop = 1;
                }
                pan[r].L = Lr; pan[r].ldl = ldl; pan[r].C = Cr; pan[r].ldcc = ldr;
            }
            if (stop) break;
        }
        if (m > 0) update(x, k, pan);
        if (abft && m > 0) {
            inject(x, (int)k, O_HOOK_UPDATE_OUT, 0, x->A, lda, x->chk, x->ldc);
            const int do_v5 = mode != 2 && (((k + 1) % x->K == 0) || (k == N - 2));   /* Opt. 3 [A14] */
            if (do_v5) {
                int stop = 0;
                for (int64_t j = k + 1; j < N && !stop; ++j)
                    for (int64_t i = j; i < N && !stop; ++i) {
                        tview_t v = gview(x, i, j, 0);
                        if (check_tile(x, &v, (int)k, O_V5, 0)) stop = 1;     /* V5 */
                    }
                if (stop) break;
            }
        }
    }
    if (abft && x->status == O_OK && g_kstop >= N) {
        inject(x, (int)N, O_HOOK_REST, 0, x->A, lda, x->chk, x->ldc);
        int stop = 0;
        for (int64_t J = 0; J < N && !stop; ++J)
            for (int64_t I = J; I < N && !stop; ++I) {
                tview_t v = gview(x, I, J, 1);
                if (check_tile(x, &v, (int)N, O_V6, 0)) stop = 1;             /* V6 */
            }
    }
    if (info) *info = x->info;
    if (nev) *nev = x->nev;
    if (chk_out) memcpy(chk_out, x->chk, sizeof(double) * (size_t)(x->ldc * n));
    if (scl_out && abft) {
        memcpy(scl_out, x->s, sizeof(double) * (size_t)n);
        memcpy(scl_out + n, x->S1, sizeof(double) * (size_t)N);
        memcpy(scl_out + n + N, x->S2, sizeof(double) * (size_t)N);
        if (x->S3) memcpy(scl_out + n + 2 * N, x->S3, sizeof(double) * (size_t)N);
    }
    free(x->chk); free(x->s); free(x->S1); free(x->S2); free(x->S3); free(rcopy); free(rchk); free(pan);
    return x->status;
}


/* ---- left-looking order: MAGMA's Alg. 1 (garbled; reading A2) with the
 * verification of Table I — NEXT-1 of SURVEY.md §8f ------------------------
 * iteration j:  SYRK  A[j,j]     -= L[j,0:j] L[j,0:j]^T        verify A (V1) and C = L[j,0:j] (V7)
 *               GEMM  A[j+1:N,j] -= L[j+1:N,0:j] L[j,0:j]^T    verify B (V2), C, D = L[j+1:N,0:j] (V7,
 *                                                               every K iterations: Opt. 3)
 *               POTF2 A[j,j] -> L[j,j]                         verify A (V5 on the updated column)
 *               TRSM  L[j+1:N,j] = A[j+1:N,j] L[j,j]^-T        verify L (V3) and B (V5)
 * Checksums: chk(A') = chk(A) - chk(LC) LC^T, chk(B') = chk(B) - chk(LD) LC^T,
 * Alg. 2, chk(LB) = chk(B') LA^-T. Online-ABFT checks results instead (V5 after the update, V3,
 * V4 after TRSM); Offline only V6. */
static int potrf_core_left(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                           int K, double c_tau, int abft, int mode, oevent_t* ev, int64_t cap,
                           int64_t* nev, int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out, int nchk) {
    octx_t X_; octx_t* x = &X_;
    memset(x, 0, sizeof *x);
    x->cnt = cnt; x->mode = mode;
    x->nchk = nchk;
    x->n = n; x->B = nb; x->N = n / nb; x->lda = lda; x->ldc = nchk * x->N > 0 ? nchk * x->N : 1;
    x->A = A; x->c_tau = c_tau > 0 ? c_tau : 64.0; x->rho = 0x1p-30;
    x->nranks = 1; x->K = K; x->correct = 1;
    x->inj = inj; x->ninj = ninj; x->ev = ev; x->cap = cap;
    if (info) *info = 0;
    if (n == 0) { if (nev) *nev = 0; return 0; }
    const int64_t N = x->N, B = nb;
    x->chk = (double*)calloc((size_t)(x->ldc * n), sizeof(double));
    x->s = (double*)malloc(sizeof(double) * (size_t)n);
    x->S1 = (double*)malloc(sizeof(double) * (size_t)N);
    x->S2 = (double*)malloc(sizeof(double) * (size_t)N);
    x->S3 = nchk == 3 ? (double*)malloc(sizeof(double) * (size_t)N) : NULL;
    double* tmp = (double*)malloc(sizeof(double) * (size_t)B);
    if (abft) { scales(x); encode(x); }
    for (int64_t j = 0; j < N && x->status == O_OK; ++j) {
        if (abft) inject(x, (int)j, O_HOOK_REST, 0, x->A, lda, x->chk, x->ldc);
        if (abft && mode == 0 && j > 0) {
            int stop = 0;
            for (int64_t p = 0; p < j && !stop; ++p)                 /* V7: C = L[j,p] and D = L[i>j,p] */
                for (int64_t i = j; i < N && !stop; ++i) {
                    if (i > j && !((j % K) == 0)) continue;          /* Opt. 3: D every K iterations */
                    tview_t v = gview(x, i, p, 1);
                    if (check_tile(x, &v, (int)j, O_V7, 0)) stop = 1;
                }
            if (stop) break;
        }
        if (abft && mode == 0 && run_checks_column(x, j, 0, O_V1, O_V2, 1)) break;   /* V1, V2 */
        if (j > 0) {   /* SYRK + GEMM: A[j:N, j] -= L[j:N, 0:j] L[j, 0:j]^T, then the checksum rows */
            const double* Lj = x->A + j * B;                          /* row block j, columns 0..jB */
            for (int64_t i = j; i < N; ++i) {
                const double* Li = x->A + i * B;
                double* T = x->A + j * B * lda + i * B;
                for (int64_t c = 0; c < B; ++c) {
                    const int64_t r0 = (i == j) ? c : 0;
                    for (int64_t r = r0; r < B; ++r) tmp[r] = 0.0;
                    for (int64_t q = 0; q < j * B; ++q) {
                        const double l = Lj[q * lda + c];
                        for (int64_t r = r0; r < B; ++r) tmp[r] += Li[q * lda + r] * l;
                    }
                    for (int64_t r = r0; r < B; ++r) T[c * lda + r] -= tmp[r];
                }
                for (int t = 0; t < nchk; ++t) {
                    const double* ck = x->chk + nchk * i + t;         /* chk(i, 0:j) row */
                    double* cd = x->chk + j * B * x->ldc + nchk * i + t;
                    for (int64_t c = 0; c < B; ++c) {
                        double a = 0.0;
                        for (int64_t q = 0; q < j * B; ++q) a += ck[q * x->ldc] * Lj[q * lda + c];
                        cd[c * x->ldc] -= a;
                    }
                }
            }
            x->cnt->flops_factor += 2.0 * (double)((N - j) * B) * B * (double)(j * B);
            x->cnt->flops_chkupd += 2.0 * nchk * (double)(N - j) * B * (double)(j * B);
        }
        if (abft) inject(x, (int)j, O_HOOK_UPDATE_OUT, 0, x->A, lda, x->chk, x->ldc);
        if (abft && mode != 2 && j > 0) {                             /* V5: the updated column j */
            int stop = 0;
            for (int64_t i = j; i < N && !stop; ++i) {
                tview_t v = gview(x, i, j, 0);
                if (check_tile(x, &v, (int)j, O_V5, 0)) stop = 1;
            }
            if (stop) break;
        }
        if (potrf_tile(x, j)) break;
        if (abft) {
            inject(x, (int)j, O_HOOK_POTRF_OUT, 0, x->A, lda, x->chk, x->ldc);
            tview_t v = gview(x, j, j, 1);
            if (mode != 2 && check_tile(x, &v, (int)j, O_V3, 0)) break;   /* V3 */
        }
        trsm_panel(x, j);
        if (abft) {
            inject(x, (int)j, O_HOOK_TRSM_OUT, 0, x->A, lda, x->chk, x->ldc);
            if (mode == 1 && run_checks_column(x, j, 1, 0, O_V4, 0)) break;  /* Online: V4 */
        }
    }
    if (abft && x->status == O_OK) {
        inject(x, (int)N, O_HOOK_REST, 0, x->A, lda, x->chk, x->ldc);
        int stop = 0;
        for (int64_t J = 0; J < N && !stop; ++J)
            for (int64_t I = J; I < N && !stop; ++I) {
                tview_t v = gview(x, I, J, 1);
                if (check_tile(x, &v, (int)N, O_V6, 0)) stop = 1;             /* V6 */
            }
    }
    if (info) *info = x->info;
    if (nev) *nev = x->nev;
    if (chk_out) memcpy(chk_out, x->chk, sizeof(double) * (size_t)(x->ldc * n));
    if (scl_out && abft) {
        memcpy(scl_out, x->s, sizeof(double) * (size_t)n);
        memcpy(scl_out + n, x->S1, sizeof(double) * (size_t)N);
        memcpy(scl_out + n + N, x->S2, sizeof(double) * (size_t)N);
    }
    if (scl_out && abft && x->S3) memcpy(scl_out + n + 2 * N, x->S3, sizeof(double) * (size_t)N);
    free(x->chk); free(x->s); free(x->S1); free(x->S2); free(x->S3); free(tmp);
    return x->status;
}

/* The factorisation with the scheme's recovery: Enhanced corrects in place; Online and Offline
 * cannot correct an error that propagated ("it needs to repeat the whole decomposition
 * again"), so an UNCORRECTABLE / NOT_SPD outcome or any detection by the final sweep re-runs the
 * factorisation once from the saved input, without the injected faults. mode 3 is the Enhanced
 * scheme with the same re-do for what two checksums cannot correct (more than one error in a
 * column of a block, P:121 [A11]): an UNCORRECTABLE outcome re-runs once.
 * Events of both runs are returned in order. */
/* prows (P>1 simulation): 2D block-cyclic process grid prows x (nranks / prows);
 * 1 = the 1D column-cyclic distribution. The arithmetic of every tile is that of one process; only
 * which rank checks a tile, and which rank's received panel copy an update reads, depend on it. */
int oracle_potrf_grid(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                      int nranks, int prows, int K, double c_tau, int abft, int mode, int order, oevent_t* ev,
                      int64_t cap, int64_t* nev, int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out,
                      int* reruns, int nchk) {
    if (n < 0) return -1;
    if (prows < 1 || nranks < 1 || nranks % prows) return -13;
    if (nchk != 2 && nchk != 3) return -12;
    if (nb < 1) return -2;
    if (n % nb) return -2;                          /* [A20] */
    if (lda < (n > 1 ? n : 1)) return -4;
    if (mode < 0 || mode > 3) return -11;
    const int redo = (mode == 3);                   /* Enhanced + re-do on UNCORRECTABLE */
    if (redo) mode = 0;
    if (nranks < 1) nranks = 1;
    if (K < 1) K = 1;
    ocount_t dummy;
    ocount_t* c = cnt ? cnt : &dummy;
    memset(c, 0, sizeof(ocount_t));
    if (reruns) *reruns = 0;
    double* A0 = NULL;
    if ((mode != 0 || redo) && n > 0) {
        A0 = (double*)malloc(sizeof(double) * (size_t)(lda * n));
        memcpy(A0, A, sizeof(double) * (size_t)(lda * n));
    }
    if (order != 0 && nranks != 1) return -7;
    int64_t nev1 = 0;
    int st = order == 0 ? potrf_core(n, nb, A, lda, inj, ninj, nranks, K, c_tau, abft, mode, ev, cap, &nev1, info, c,
                                     chk_out, scl_out, nchk, prows)
                        : potrf_core_left(n, nb, A, lda, inj, ninj, K, c_tau, abft, mode, ev, cap, &nev1, info, c,
                                          chk_out, scl_out, nchk);
    /* Online / Offline: a detection at the final sweep means an error escaped the scheme's
     * online checks and may have propagated -> re-do. */
    int v6_detect = 0;
    for (int64_t e = 0; ev && e < nev1 && e < cap; ++e) v6_detect |= (ev[e].check == O_V6);
    if ((mode != 0 && (st == O_STATUS_UNCORRECTABLE || st == O_STATUS_NOT_SPD || v6_detect)) ||
        (redo && st == O_STATUS_UNCORRECTABLE)) {
        memcpy(A, A0, sizeof(double) * (size_t)(lda * n));
        int64_t nev2 = 0;
        const int64_t off = nev1 < cap ? nev1 : cap;
        st = order == 0 ? potrf_core(n, nb, A, lda, NULL, 0, nranks, K, c_tau, abft, mode, ev ? ev + off : NULL,
                                     cap - off, &nev2, info, c, chk_out, scl_out, nchk, prows)
                        : potrf_core_left(n, nb, A, lda, NULL, 0, K, c_tau, abft, mode, ev ? ev + off : NULL,
                                          cap - off, &nev2, info, c, chk_out, scl_out, nchk);
        nev1 += nev2;
        if (reruns) *reruns = 1;
    }
    free(A0);
    if (nev) *nev = nev1;
    return st;
}

int oracle_potrf_nchk(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                      int nranks, int K, double c_tau, int abft, int mode, int order, oevent_t* ev, int64_t cap,
                      int64_t* nev, int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out,
                      int* reruns, int nchk) {
    return oracle_potrf_grid(n, nb, A, lda, inj, ninj, nranks < 1 ? 1 : nranks, 1, K, c_tau, abft, mode, order, ev,
                             cap, nev, info, cnt, chk_out, scl_out, reruns, nchk);
}

int oracle_potrf_mode(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                      int nranks, int K, double c_tau, int abft, int mode, int order, oevent_t* ev, int64_t cap,
                      int64_t* nev, int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out,
                      int* reruns) {
    return oracle_potrf_nchk(n, nb, A, lda, inj, ninj, nranks, K, c_tau, abft, mode, order, ev, cap, nev, info, cnt,
                             chk_out, scl_out, reruns, 2);
}

int oracle_potrf(int64_t n, int64_t nb, double* A, int64_t lda, const oinj_t* inj, int64_t ninj,
                 int nranks, int K, double c_tau, int abft, oevent_t* ev, int64_t cap, int64_t* nev,
                 int64_t* info, ocount_t* cnt, double* chk_out, double* scl_out) {
    return oracle_potrf_mode(n, nb, A, lda, inj, ninj, nranks, K, c_tau, abft, 0, 0, ev, cap, nev, info, cnt,
                             chk_out, scl_out, NULL);
}

/* ---- stand-alone steps for kernel-level parity tests ----------------------------------- */

/* abft_encode semantics: chk (2N x n, ldc) and scales = [s (n) | S1 (N) | S2 (N)]. */
int oracle_encode(int64_t n, int64_t nb, const double* A, int64_t lda, double* chk, int64_t ldc, double* scl) {
    if (n < 0) return -1;
    if (nb < 1 || n % nb) return -2;
    if (lda < (n > 1 ? n : 1)) return -4;
    octx_t X_; octx_t* x = &X_; memset(x, 0, sizeof *x);
    ocount_t c; memset(&c, 0, sizeof c); x->cnt = &c;
    x->n = n; x->B = nb; x->N = n / nb; x->lda = lda; x->ldc = ldc; x->nchk = 2;
    x->A = (double*)A; x->chk = chk; x->s = scl; x->S1 = scl + n; x->S2 = scl + n + x->N;
    x->nranks = 1;
    if (n == 0) return 0;
    scales(x); encode(x);
    return 0;
}

/* abft_verify semantics: check every lower tile (I >= J) once, factored or not; correct if
 * asked. Returns status (0 / 1 UNCORRECTABLE); events as in oracle_potrf (k = -1, V = 6 if
 * factored else 5). Used by tests to pin the detector alone. */
int oracle_verify(int64_t n, int64_t nb, double* A, int64_t lda, double* chk, int64_t ldc, const double* scl,
                  int factored, int correct, double c_tau, oevent_t* ev, int64_t cap, int64_t* nev, ocount_t* cnt) {
    if (n < 0) return -1;
    if (nb < 1 || n % nb) return -2;
    octx_t X_; octx_t* x = &X_; memset(x, 0, sizeof *x);
    ocount_t c0; memset(&c0, 0, sizeof c0);
    x->cnt = cnt ? cnt : &c0; memset(x->cnt, 0, sizeof(ocount_t));
    x->n = n; x->B = nb; x->N = n / nb; x->lda = lda; x->ldc = ldc; x->nchk = 2;
    x->A = A; x->chk = chk; x->s = (double*)scl; x->S1 = (double*)scl + n; x->S2 = (double*)scl + n + x->N;
    x->c_tau = c_tau > 0 ? c_tau : 64.0; x->rho = 0x1p-30; x->correct = correct;
    x->ev = ev; x->cap = cap; x->nranks = 1;
    for (int64_t J = 0; J < x->N; ++J)
        for (int64_t I = J; I < x->N; ++I) {
            tview_t v = gview(x, I, J, factored);
            if (check_tile(x, &v, -1, factored ? O_V6 : O_V5, 0)) goto done;
        }
done:
    if (nev) *nev = x->nev;
    return x->status;
}

/* Bounded sample for timing (bench.py's cpu_baseline / reference arm on large n): the
 * Enhanced right-looking factorisation stopped after kstop iterations. Returns the status;
 * cnt receives the work done (flops of the iterations run), so that the caller can extrapolate
 * the whole factorisation's time by flops. */
int oracle_potrf_prefix(int64_t n, int64_t nb, double* A, int64_t lda, int64_t kstop, ocount_t* cnt) {
    if (n < 0) return -1;
    if (nb < 1 || n % nb) return -2;
    if (lda < (n > 1 ? n : 1)) return -4;
    ocount_t dummy;
    ocount_t* c = cnt ? cnt : &dummy;
    memset(c, 0, sizeof(ocount_t));
    int64_t nev = 0, info = 0;
    g_kstop = kstop < 0 ? 0 : kstop;
    const int st = potrf_core(n, nb, A, lda, NULL, 0, 1, 1, 64.0, 1, 0, NULL, 0, &nev, &info, c, NULL, NULL, 2, 1);
    g_kstop = INT64_MAX;
    return st;
}

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
