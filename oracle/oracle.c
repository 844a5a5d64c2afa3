/*
 * oracle.c -- plain, slow CPU reference for the G1 MSM.
 *
 *   TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 *   bench.py's cpu_baseline / --impl reference legs may load this library.
 *   It shares no code, header, table or constant with the CUDA product path
 *   (paper_conf_asplos_maxsm0k0zsh23_b200/csrc); curve constants are passed
 *   in by the caller (oracle/curves.py holds the oracle's own copy).
 *
 * What it computes is the definition (§2.1):
 *     Q = sum_{i<n} k_i (x) P_i      over E(F_p): y^2 = x^3 + a x + b
 *
 *   1. bignum: u32 limbs, schoolbook products, remainder by Knuth's
 *      Algorithm D (TAOCP 4.3.1).  No Montgomery form.
 *   2. field inverse: the binary extended Euclidean algorithm (HAC 14.61,
 *      specialised to an odd modulus).
 *   3. group law: AFFINE chord-and-tangent formulas with every exceptional
 *      case explicit (O, P == Q, P == -Q); "PADD ... including point doubling"
 *      (PAPER.md:116 fn. 2).
 *   4. PMUL: left-to-right binary double-and-add.
 *   5. MSM: each thread sums k_i P_i over a contiguous chunk; the chunk sums
 *      are added in chunk order.  The group is abelian and exact, so the
 *      result is independent of the order.
 *
 * G2 (the MSM optimisations "apply to both G1 and G2") is the
 * same definition over F_p^2 = F_p[u]/(u^2 - beta): an element is c0 + c1 u,
 * stored c0 || c1, and its product is the schoolbook polynomial product
 * reduced by u^2 = beta (no Karatsuba: plain definition).
 *
 * Encoding: a point is 2D little-endian u32 limbs x || y (D = deg * L limbs
 * per coordinate), canonical (< p per F_p coordinate); the identity O is
 * (0,0).  A scalar is Ls little-endian u32 limbs, any integer (not reduced
 * mod r).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define MAXL 24

typedef struct {
    int L;               /* limbs of one F_p coordinate in the encoding */
    int Le;              /* effective limbs of p (top limb nonzero) */
    int deg;             /* 1: E(F_p) (G1); 2: E'(F_p^2) (G2, the twist) */
    int D;               /* limbs of one curve coordinate = deg * L */
    uint32_t p[MAXL];
    uint32_t beta[MAXL]; /* deg 2: F_p^2 = F_p[u] / (u^2 - beta) */
    uint32_t a[2 * MAXL];/* curve coefficient a, deg coordinates */
} fctx;

typedef struct {
    uint32_t x[2 * MAXL], y[2 * MAXL];
    int inf;             /* 1 = identity O */
} apt;

/* ------------------------------------------------------------------ bignum */

static int bn_cmp(const uint32_t *x, const uint32_t *y, int n) {
    for (int i = n - 1; i >= 0; --i) {
        if (x[i] != y[i]) return x[i] > y[i] ? 1 : -1;
    }
    return 0;
}

static int bn_is_zero(const uint32_t *x, int n) {
    for (int i = 0; i < n; ++i)
        if (x[i]) return 0;
    return 1;
}

static int bn_is_one(const uint32_t *x, int n) {
    if (x[0] != 1) return 0;
    for (int i = 1; i < n; ++i)
        if (x[i]) return 0;
    return 1;
}

static uint32_t bn_add(uint32_t *r, const uint32_t *x, const uint32_t *y, int n) {
    uint64_t c = 0;
    for (int i = 0; i < n; ++i) {
        c += (uint64_t)x[i] + y[i];
        r[i] = (uint32_t)c;
        c >>= 32;
    }
    return (uint32_t)c;
}

static uint32_t bn_sub(uint32_t *r, const uint32_t *x, const uint32_t *y, int n) {
    int64_t b = 0;
    for (int i = 0; i < n; ++i) {
        int64_t t = (int64_t)x[i] - y[i] + b;
        r[i] = (uint32_t)t;
        b = t >> 32;            /* 0 or -1 */
    }
    return (uint32_t)(b & 1);
}

/* x >>= 1, shifting `top` in as the new most significant bit */
static void bn_shr1(uint32_t *x, int n, uint32_t top) {
    for (int i = 0; i < n - 1; ++i) x[i] = (x[i] >> 1) | (x[i + 1] << 31);
    x[n - 1] = (x[n - 1] >> 1) | (top << 31);
}

/* schoolbook product: t[0..2n) = x * y */
static void bn_mul(uint32_t *t, const uint32_t *x, const uint32_t *y, int n) {
    memset(t, 0, sizeof(uint32_t) * 2 * n);
    for (int i = 0; i < n; ++i) {
        uint64_t c = 0;
        for (int j = 0; j < n; ++j) {
            c += (uint64_t)x[i] * y[j] + t[i + j];
            t[i + j] = (uint32_t)c;
            c >>= 32;
        }
        t[i + n] = (uint32_t)c;
    }
}

/* Knuth Algorithm D remainder: r[0..n) = u[0..m) mod v[0..n), v[n-1] != 0, m >= n */
static void bn_mod(uint32_t *r, const uint32_t *u, int m, const uint32_t *v, int n) {
    if (n == 1) {
        uint64_t rem = 0;
        for (int i = m - 1; i >= 0; --i) rem = ((rem << 32) | u[i]) % v[0];
        r[0] = (uint32_t)rem;
        return;
    }
    uint32_t un[2 * MAXL + 1], vn[MAXL];
    int s = __builtin_clz(v[n - 1]);
    for (int i = n - 1; i > 0; --i)
        vn[i] = (v[i] << s) | (s ? (uint32_t)((uint64_t)v[i - 1] >> (32 - s)) : 0);
    vn[0] = v[0] << s;
    un[m] = s ? (uint32_t)((uint64_t)u[m - 1] >> (32 - s)) : 0;
    for (int i = m - 1; i > 0; --i)
        un[i] = (u[i] << s) | (s ? (uint32_t)((uint64_t)u[i - 1] >> (32 - s)) : 0);
    un[0] = u[0] << s;

    const uint64_t B = 1ull << 32;
    for (int j = m - n; j >= 0; --j) {
        uint64_t num = ((uint64_t)un[j + n] << 32) | un[j + n - 1];
        uint64_t qhat = num / vn[n - 1];
        uint64_t rhat = num % vn[n - 1];
        while (qhat >= B || qhat * vn[n - 2] > ((rhat << 32) | un[j + n - 2])) {
            qhat--;
            rhat += vn[n - 1];
            if (rhat >= B) break;
        }
        /* multiply and subtract */
        int64_t borrow = 0;
        uint64_t carry = 0;
        for (int i = 0; i < n; ++i) {
            uint64_t prod = qhat * vn[i] + carry;
            carry = prod >> 32;
            int64_t t = (int64_t)un[i + j] - (int64_t)(uint32_t)prod + borrow;
            un[i + j] = (uint32_t)t;
            borrow = t >> 32;
        }
        int64_t t = (int64_t)un[j + n] - (int64_t)carry + borrow;
        un[j + n] = (uint32_t)t;
        if (t < 0) {            /* qhat was one too large: add v back */
            uint64_t c = 0;
            for (int i = 0; i < n; ++i) {
                c += (uint64_t)un[i + j] + vn[i];
                un[i + j] = (uint32_t)c;
                c >>= 32;
            }
            un[j + n] += (uint32_t)c;
        }
    }
    for (int i = 0; i < n; ++i)
        r[i] = (un[i] >> s) | (s ? (uint32_t)((uint64_t)un[i + 1] << (32 - s)) : 0);
}

/* ------------------------------------------------------------------- F_p */

static void fp_add(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    uint32_t t[MAXL];
    uint32_t c = bn_add(t, x, y, f->L);
    if (c || bn_cmp(t, f->p, f->L) >= 0) bn_sub(t, t, f->p, f->L);
    memcpy(r, t, sizeof(uint32_t) * f->L);
}

static void fp_sub(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    uint32_t t[MAXL];
    if (bn_sub(t, x, y, f->L)) bn_add(t, t, f->p, f->L);
    memcpy(r, t, sizeof(uint32_t) * f->L);
}

static void fp_mul(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    uint32_t t[2 * MAXL], q[MAXL];
    bn_mul(t, x, y, f->L);
    memset(q, 0, sizeof(q));
    bn_mod(q, t, 2 * f->L, f->p, f->Le);
    memcpy(r, q, sizeof(uint32_t) * f->L);
}

/* (x + p) / 2 or x / 2 modulo p, for x in [0, p) */
static void fp_half(const fctx *f, uint32_t *x) {
    if (x[0] & 1) {
        uint32_t c = bn_add(x, x, f->p, f->L);
        bn_shr1(x, f->L, c);
    } else {
        bn_shr1(x, f->L, 0);
    }
}

/* binary extended Euclid (HAC 14.61 for odd p); x != 0 required */
static void fp_inv(const fctx *f, uint32_t *r, const uint32_t *x) {
    int L = f->L;
    uint32_t u[MAXL], v[MAXL], x1[MAXL], x2[MAXL];
    memcpy(u, x, sizeof(uint32_t) * L);
    memcpy(v, f->p, sizeof(uint32_t) * L);
    memset(x1, 0, sizeof(x1));
    memset(x2, 0, sizeof(x2));
    x1[0] = 1;
    while (!bn_is_one(u, L) && !bn_is_one(v, L)) {
        while (!(u[0] & 1)) { bn_shr1(u, L, 0); fp_half(f, x1); }
        while (!(v[0] & 1)) { bn_shr1(v, L, 0); fp_half(f, x2); }
        if (bn_cmp(u, v, L) >= 0) {
            bn_sub(u, u, v, L);
            fp_sub(f, x1, x1, x2);
        } else {
            bn_sub(v, v, u, L);
            fp_sub(f, x2, x2, x1);
        }
    }
    memcpy(r, bn_is_one(u, L) ? x1 : x2, sizeof(uint32_t) * L);
}

/* --------------------------------------------- F_p^deg (deg = 1 or 2) */
/* An element is deg F_p coordinates; for deg 2, c0 + c1 u with u^2 = beta. */

static void fe_add(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    for (int i = 0; i < f->deg; ++i) fp_add(f, r + i * f->L, x + i * f->L, y + i * f->L);
}

static void fe_sub(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    for (int i = 0; i < f->deg; ++i) fp_sub(f, r + i * f->L, x + i * f->L, y + i * f->L);
}

/* (x0 + x1 u)(y0 + y1 u) = (x0 y0 + beta x1 y1) + (x0 y1 + x1 y0) u */
static void fe_mul(const fctx *f, uint32_t *r, const uint32_t *x, const uint32_t *y) {
    if (f->deg == 1) { fp_mul(f, r, x, y); return; }
    int L = f->L;
    uint32_t t0[MAXL], t1[MAXL], t2[MAXL], r0[MAXL], r1[MAXL];
    fp_mul(f, t0, x, y);                 /* x0 y0 */
    fp_mul(f, t1, x + L, y + L);         /* x1 y1 */
    fp_mul(f, t2, f->beta, t1);          /* beta x1 y1 */
    fp_add(f, r0, t0, t2);
    fp_mul(f, t0, x, y + L);             /* x0 y1 */
    fp_mul(f, t1, x + L, y);             /* x1 y0 */
    fp_add(f, r1, t0, t1);
    memcpy(r, r0, sizeof(uint32_t) * L);
    memcpy(r + L, r1, sizeof(uint32_t) * L);
}

/* 1 / (x0 + x1 u) = (x0 - x1 u) / (x0^2 - beta x1^2); x != 0 required */
static void fe_inv(const fctx *f, uint32_t *r, const uint32_t *x) {
    if (f->deg == 1) { fp_inv(f, r, x); return; }
    int L = f->L;
    uint32_t t0[MAXL], t1[MAXL], nrm[MAXL], ni[MAXL], zero[MAXL];
    memset(zero, 0, sizeof(zero));
    fp_mul(f, t0, x, x);
    fp_mul(f, t1, x + L, x + L);
    fp_mul(f, t1, f->beta, t1);
    fp_sub(f, nrm, t0, t1);              /* the norm, in F_p */
    fp_inv(f, ni, nrm);
    fp_mul(f, t0, x, ni);
    fp_sub(f, t1, zero, x + L);
    fp_mul(f, t1, t1, ni);
    memcpy(r, t0, sizeof(uint32_t) * L);
    memcpy(r + L, t1, sizeof(uint32_t) * L);
}

/* ------------------------------------------------------------ group law */

static void ec_add(const fctx *f, apt *R, const apt *P, const apt *Q) {
    int D = f->D;
    if (P->inf) { *R = *Q; return; }
    if (Q->inf) { *R = *P; return; }
    uint32_t lam[2 * MAXL], num[2 * MAXL], den[2 * MAXL], t[2 * MAXL];
    if (bn_cmp(P->x, Q->x, D) == 0) {
        fe_add(f, t, P->y, Q->y);
        if (bn_is_zero(t, D)) {             /* P == -Q */
            memset(R, 0, sizeof(*R));
            R->inf = 1;
            return;
        }
        /* tangent: lam = (3 x^2 + a) / (2 y) */
        fe_mul(f, t, P->x, P->x);
        fe_add(f, num, t, t);
        fe_add(f, num, num, t);
        fe_add(f, num, num, f->a);
        fe_add(f, den, P->y, P->y);
    } else {
        /* chord: lam = (y2 - y1) / (x2 - x1) */
        fe_sub(f, num, Q->y, P->y);
        fe_sub(f, den, Q->x, P->x);
    }
    fe_inv(f, t, den);
    fe_mul(f, lam, num, t);
    uint32_t x3[2 * MAXL], y3[2 * MAXL];
    fe_mul(f, x3, lam, lam);
    fe_sub(f, x3, x3, P->x);
    fe_sub(f, x3, x3, Q->x);
    fe_sub(f, t, P->x, x3);
    fe_mul(f, y3, lam, t);
    fe_sub(f, y3, y3, P->y);
    memset(R, 0, sizeof(*R));
    memcpy(R->x, x3, sizeof(uint32_t) * D);
    memcpy(R->y, y3, sizeof(uint32_t) * D);
    R->inf = 0;
}

/* left-to-right double-and-add over the Ls-limb scalar k */
static void ec_mul(const fctx *f, apt *R, const uint32_t *k, int Ls, const apt *P) {
    apt acc;
    memset(&acc, 0, sizeof(acc));
    acc.inf = 1;
    for (int i = 32 * Ls - 1; i >= 0; --i) {
        apt t;
        ec_add(f, &t, &acc, &acc);
        acc = t;
        if ((k[i / 32] >> (i % 32)) & 1) {
            ec_add(f, &t, &acc, P);
            acc = t;
        }
    }
    *R = acc;
}

static void load_point(const fctx *f, apt *P, const uint32_t *src) {
    memset(P, 0, sizeof(*P));
    memcpy(P->x, src, sizeof(uint32_t) * f->D);
    memcpy(P->y, src + f->D, sizeof(uint32_t) * f->D);
    P->inf = bn_is_zero(P->x, f->D) && bn_is_zero(P->y, f->D);
}

static void store_point(const fctx *f, uint32_t *dst, const apt *P) {
    if (P->inf) {
        memset(dst, 0, sizeof(uint32_t) * 2 * f->D);
        return;
    }
    memcpy(dst, P->x, sizeof(uint32_t) * f->D);
    memcpy(dst + f->D, P->y, sizeof(uint32_t) * f->D);
}

/* deg 1: beta unused (may be NULL); a has deg * L limbs */
static int init_ctx(fctx *f, int L, int deg, const uint32_t *p, const uint32_t *beta, const uint32_t *a) {
    if (L < 1 || L > MAXL || (deg != 1 && deg != 2)) return -1;
    memset(f, 0, sizeof(*f));
    f->L = L;
    f->deg = deg;
    f->D = deg * L;
    memcpy(f->p, p, sizeof(uint32_t) * L);
    if (deg == 2) memcpy(f->beta, beta, sizeof(uint32_t) * L);
    memcpy(f->a, a, sizeof(uint32_t) * f->D);
    f->Le = L;
    while (f->Le > 1 && f->p[f->Le - 1] == 0) f->Le--;
    if (!(f->p[0] & 1)) return -1;
    return 0;
}

/* ------------------------------------------------------------- threading */

typedef struct {
    const fctx *f;
    const uint32_t *points, *scalars;
    int Ls;
    uint64_t begin, end;
    uint32_t *out;         /* msm: one point; mul_each: n points */
    int each;
} job;

static void *run_job(void *arg) {
    job *j = (job *)arg;
    const fctx *f = j->f;
    apt acc;
    memset(&acc, 0, sizeof(acc));
    acc.inf = 1;
    for (uint64_t i = j->begin; i < j->end; ++i) {
        apt P, R;
        const uint32_t *k = j->scalars + (size_t)i * j->Ls;
        load_point(f, &P, j->points + (j->each ? 0 : (size_t)i * 2 * f->D));
        if (P.inf || bn_is_zero(k, j->Ls)) {
            memset(&R, 0, sizeof(R));
            R.inf = 1;
        } else {
            ec_mul(f, &R, k, j->Ls, &P);
        }
        if (j->each) {
            store_point(f, j->out + (size_t)i * 2 * f->D, &R);
        } else {
            apt t;
            ec_add(f, &t, &acc, &R);
            acc = t;
        }
    }
    if (!j->each) store_point(f, j->out, &acc);
    return NULL;
}

static int run_parallel(const fctx *f, const uint32_t *points, const uint32_t *scalars, int Ls,
                        uint64_t n, uint32_t *out, int nthreads, int each) {
    if (nthreads < 1) nthreads = 1;
    if ((uint64_t)nthreads > n) nthreads = n ? (int)n : 1;
    job *jobs = (job *)calloc(nthreads, sizeof(job));
    pthread_t *th = (pthread_t *)calloc(nthreads, sizeof(pthread_t));
    uint32_t *partial = (uint32_t *)calloc((size_t)nthreads * 2 * f->D, sizeof(uint32_t));
    if (!jobs || !th || !partial) { free(jobs); free(th); free(partial); return -2; }
    uint64_t chunk = (n + nthreads - 1) / nthreads;
    for (int t = 0; t < nthreads; ++t) {
        jobs[t].f = f;
        jobs[t].points = points;
        jobs[t].scalars = scalars;
        jobs[t].Ls = Ls;
        jobs[t].begin = (uint64_t)t * chunk < n ? (uint64_t)t * chunk : n;
        jobs[t].end = (uint64_t)(t + 1) * chunk < n ? (uint64_t)(t + 1) * chunk : n;
        jobs[t].out = each ? out : partial + (size_t)t * 2 * f->D;
        jobs[t].each = each;
        pthread_create(&th[t], NULL, run_job, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    if (!each) {
        apt acc, P, s;
        memset(&acc, 0, sizeof(acc));
        acc.inf = 1;
        for (int t = 0; t < nthreads; ++t) {
            load_point(f, &P, partial + (size_t)t * 2 * f->D);
            ec_add(f, &s, &acc, &P);
            acc = s;
        }
        store_point(f, out, &acc);
    }
    free(jobs);
    free(th);
    free(partial);
    return 0;
}

/* ------------------------------------------------------------- exports */

/* Q = sum k_i P_i over E(F_p^deg).  points: n x 2 deg L limbs; scalars: n x Ls
 * limbs; out: 2 deg L limbs.  beta: deg 2 only (u^2 = beta); a: deg L limbs. */
int oracle_msm_ext(int L, int deg, const uint32_t *p, const uint32_t *beta, const uint32_t *a,
                   const uint32_t *points, const uint32_t *scalars, int Ls, uint64_t n, uint32_t *out,
                   int nthreads) {
    fctx f;
    if (init_ctx(&f, L, deg, p, beta, a)) return -1;
    return run_parallel(&f, points, scalars, Ls, n, out, nthreads, 0);
}

/* out_i = k_i P for one base point P; out: n points. */
int oracle_mul_each_ext(int L, int deg, const uint32_t *p, const uint32_t *beta, const uint32_t *a,
                        const uint32_t *P, const uint32_t *scalars, int Ls, uint64_t n, uint32_t *out,
                        int nthreads) {
    fctx f;
    if (init_ctx(&f, L, deg, p, beta, a)) return -1;
    return run_parallel(&f, P, scalars, Ls, n, out, nthreads, 1);
}

/* R = P + Q (affine, explicit cases) */
int oracle_ec_add_ext(int L, int deg, const uint32_t *p, const uint32_t *beta, const uint32_t *a,
                      const uint32_t *P, const uint32_t *Q, uint32_t *R) {
    fctx f;
    if (init_ctx(&f, L, deg, p, beta, a)) return -1;
    apt A, B, C;
    load_point(&f, &A, P);
    load_point(&f, &B, Q);
    ec_add(&f, &C, &A, &B);
    store_point(&f, R, &C);
    return 0;
}

/* G1 forms (deg 1) */
int oracle_msm(int L, const uint32_t *p, const uint32_t *a, const uint32_t *points,
               const uint32_t *scalars, int Ls, uint64_t n, uint32_t *out, int nthreads) {
    return oracle_msm_ext(L, 1, p, NULL, a, points, scalars, Ls, n, out, nthreads);
}

int oracle_mul_each(int L, const uint32_t *p, const uint32_t *a, const uint32_t *P,
                    const uint32_t *scalars, int Ls, uint64_t n, uint32_t *out, int nthreads) {
    return oracle_mul_each_ext(L, 1, p, NULL, a, P, scalars, Ls, n, out, nthreads);
}

int oracle_ec_add(int L, const uint32_t *p, const uint32_t *a, const uint32_t *P,
                  const uint32_t *Q, uint32_t *R) {
    return oracle_ec_add_ext(L, 1, p, NULL, a, P, Q, R);
}

/* r = x * y in F_p^2 (u^2 = beta), exported for the field pins */
int oracle_fp2_mul(int L, const uint32_t *p, const uint32_t *beta, const uint32_t *x, const uint32_t *y,
                   uint32_t *r) {
    fctx f;
    uint32_t zero[2 * MAXL] = {0};
    if (init_ctx(&f, L, 2, p, beta, zero)) return -1;
    fe_mul(&f, r, x, y);
    return 0;
}

int oracle_fp_mul(int L, const uint32_t *p, const uint32_t *x, const uint32_t *y, uint32_t *r) {
    fctx f;
    uint32_t zero[MAXL] = {0};
    if (init_ctx(&f, L, 1, p, NULL, zero)) return -1;
    fp_mul(&f, r, x, y);
    return 0;
}

int oracle_fp_inv(int L, const uint32_t *p, const uint32_t *x, uint32_t *r) {
    fctx f;
    uint32_t zero[MAXL] = {0};
    if (init_ctx(&f, L, 1, p, NULL, zero)) return -1;
    if (bn_is_zero(x, L)) return -3;
    fp_inv(&f, r, x);
    return 0;
}

/* ------------------------------------------------ NTT definition (NEXT-4) */
/* a_k = A(x_k) = sum_i A_i x_k^i over F_r by Horner's rule (PAPER.md:128
 * §2.2: the N-NTT is the evaluation of A at the powers of w_N).  One output
 * per call of horner(); threads split the evaluation points. */
typedef struct {
    const fctx *f;
    const uint32_t *coeffs, *xs;
    uint64_t n;
    int begin, end;
    uint32_t *out;
} ejob;

static void *run_eval(void *arg) {
    ejob *j = (ejob *)arg;
    const fctx *f = j->f;
    int L = f->L;
    for (int q = j->begin; q < j->end; ++q) {
        uint32_t acc[MAXL];
        memset(acc, 0, sizeof(acc));
        for (uint64_t i = j->n; i-- > 0;) {
            fp_mul(f, acc, acc, j->xs + (size_t)q * L);
            fp_add(f, acc, acc, j->coeffs + (size_t)i * L);
        }
        memcpy(j->out + (size_t)q * L, acc, sizeof(uint32_t) * L);
    }
    return NULL;
}

/* out[q] = A(xs[q]) mod r, q < m; coeffs: n x L limbs (< r), xs: m x L limbs */
int oracle_poly_eval(int L, const uint32_t *r, const uint32_t *coeffs, uint64_t n, const uint32_t *xs,
                     int m, uint32_t *out, int nthreads) {
    fctx f;
    uint32_t zero[MAXL] = {0};
    if (init_ctx(&f, L, 1, r, NULL, zero)) return -1;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > m) nthreads = m > 0 ? m : 1;
    ejob *jobs = (ejob *)calloc(nthreads, sizeof(ejob));
    pthread_t *th = (pthread_t *)calloc(nthreads, sizeof(pthread_t));
    if (!jobs || !th) { free(jobs); free(th); return -2; }
    int chunk = (m + nthreads - 1) / nthreads;
    for (int t = 0; t < nthreads; ++t) {
        jobs[t].f = &f;
        jobs[t].coeffs = coeffs;
        jobs[t].xs = xs;
        jobs[t].n = n;
        jobs[t].begin = t * chunk < m ? t * chunk : m;
        jobs[t].end = (t + 1) * chunk < m ? (t + 1) * chunk : m;
        jobs[t].out = out;
        pthread_create(&th[t], NULL, run_eval, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(jobs);
    free(th);
    return 0;
}

/* r = u mod v (Knuth D), exported so the tests can pin it against Python ints */
int oracle_bn_mod(const uint32_t *u, int m, const uint32_t *v, int n, uint32_t *r) {
    if (n < 1 || n > MAXL || m < n || m > 2 * MAXL || v[n - 1] == 0) return -1;
    bn_mod(r, u, m, v, n);
    return 0;
}
