/* oracle/trid_oracle.c — TEST INFRASTRUCTURE ONLY.  See trid_oracle.h for the contract.
 *
 * Plain CPU reference for Wang et al., PPoPP'25 (PAPER.md = P:<line>).  Every routine is written in
 * the paper's order and notation with no blocking, fusion or reordering beyond what the cited
 * passage states.  It never includes or links anything from the CUDA library.
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py
 * against LAPACK special cases, closed forms, brute force or invariants; none is "parity unpinned".
 */
#include "trid_oracle.h"

#include <float.h>
#include <math.h>
#include <stdlib.h>
#include <string.h>

#define AT(X, i, j, ld) (X)[(size_t)(j) * (size_t)(ld) + (size_t)(i)]

static double* zalloc(size_t cnt) {
  double* p = (double*)calloc(cnt ? cnt : 1, sizeof(double));
  if (!p) abort();
  return p;
}

/* ---------------------------------------------------------------------------------------------
 * P:86-88 Householder: H(v) x = ||x|| e1.  Reading R1 fixes the sign/scaling as LAPACK dlarfg:
 * beta = -sign(alpha) sqrt(alpha^2 + sigma) (sign taken from the sign bit, R1'), v = x / (alpha - beta) with v0 = 1,
 * tau = (beta - alpha) / beta; sigma == 0 -> tau = 0, beta = alpha (no reflection).
 * ------------------------------------------------------------------------------------------- */
double oracle_house(int64_t len, double* x, int64_t incx, double* beta) {
  if (len <= 0) { *beta = 0.0; return 0.0; }
  double alpha = x[0];
  if (len == 1) { *beta = alpha; return 0.0; }
  double sigma = 0.0;
  for (int64_t i = 1; i < len; ++i) sigma += x[i * incx] * x[i * incx];
  if (sigma == 0.0) { *beta = alpha; return 0.0; }
  double nrm = sqrt(alpha * alpha + sigma);
  double bt = signbit(alpha) ? nrm : -nrm; /* R1': sign bit, as LAPACK's SIGN(): alpha = -0.0 -> beta > 0 */
  double tau = (bt - alpha) / bt;
  double scal = 1.0 / (alpha - bt);
  for (int64_t i = 1; i < len; ++i) x[i * incx] *= scal;
  *beta = bt;
  return tau;
}

/* Symmetric (lower-referenced) element accessor. */
static inline double sym_get(const double* A, int64_t lda, int64_t i, int64_t j) {
  return i >= j ? AT(A, i, j, lda) : AT(A, j, i, lda);
}

/* Two-sided rank-2 update of the trailing symmetric block A(o:n, o:n) by H = I - tau v v^T
 * (v has length n-o, v[0] = 1): p = tau A v; w = p - 1/2 tau (p^T v) v; A -= v w^T + w v^T (lower).
 * This is the textbook dsytd2 / sec. 2.3 trailing update (P:125 with one reflector). */
static void two_sided_rank2(int64_t n, int64_t o, double* A, int64_t lda, const double* v, double tau) {
  int64_t m = n - o;
  double* p = zalloc((size_t)m);
  for (int64_t i = 0; i < m; ++i) {
    double s = 0.0;
    for (int64_t j = 0; j < m; ++j) s += sym_get(A, lda, o + i, o + j) * v[j];
    p[i] = tau * s;
  }
  double pv = 0.0;
  for (int64_t i = 0; i < m; ++i) pv += p[i] * v[i];
  double alpha = -0.5 * tau * pv;
  for (int64_t i = 0; i < m; ++i) p[i] += alpha * v[i]; /* p is now w */
  for (int64_t j = 0; j < m; ++j)
    for (int64_t i = j; i < m; ++i) AT(A, o + i, o + j, lda) -= v[i] * p[j] + p[i] * v[j];
  free(p);
}

/* O1: LAPACK dsytd2 (uplo = 'L'), one Householder per column (sec. 2.2). */
void oracle_sytd2(int64_t n, double* A, int64_t lda, double* d, double* e, double* tau) {
  if (n <= 0) return;
  double* v = zalloc((size_t)n);
  for (int64_t i = 0; i + 1 < n; ++i) {
    int64_t len = n - i - 1;
    double beta;
    double taui = oracle_house(len, &AT(A, i + 1, i, lda), 1, &beta);
    e[i] = beta;
    if (taui != 0.0) {
      v[0] = 1.0;
      for (int64_t r = 1; r < len; ++r) v[r] = AT(A, i + 1 + r, i, lda);
      two_sided_rank2(n, i + 1, A, lda, v, taui);
    }
    AT(A, i + 1, i, lda) = beta;
    d[i] = AT(A, i, i, lda);
    tau[i] = taui;
  }
  d[n - 1] = AT(A, n - 1, n - 1, lda);
  free(v);
}

/* O2a: naive SBR to bandwidth b (sec. 2.3, Fig. 2): the panel QR and the ZY trailing update of
 * P:123-127 taken one reflector at a time.  Column c's reflector acts on rows c+b..n-1. */
void oracle_sbr_naive(int64_t n, int64_t b, double* A, int64_t lda, double* tau1) {
  for (int64_t c = 0; c < n; ++c) tau1[c] = 0.0;
  if (n <= 0 || b < 1) return;
  double* v = zalloc((size_t)n);
  for (int64_t c = 0; c + b + 1 < n; ++c) { /* c <= n-b-2 */
    int64_t o = c + b, len = n - o;
    double beta;
    double tau = oracle_house(len, &AT(A, o, c, lda), 1, &beta);
    tau1[c] = tau;
    if (tau != 0.0) {
      v[0] = 1.0;
      for (int64_t r = 1; r < len; ++r) v[r] = AT(A, o + r, c, lda);
      /* left-apply to the remaining columns of the panel that are not part of the trailing matrix */
      for (int64_t j = c + 1; j < o && j < n; ++j) {
        double s = 0.0;
        for (int64_t r = 0; r < len; ++r) s += v[r] * AT(A, o + r, j, lda);
        s *= tau;
        for (int64_t r = 0; r < len; ++r) AT(A, o + r, j, lda) -= s * v[r];
      }
      two_sided_rank2(n, o, A, lda, v, tau);
    }
    AT(A, o, c, lda) = beta;
  }
  free(v);
}

/* Householder QR of a panel ("QR(Panel) = (I - W Y^T) R"), column by column. */
void oracle_panel_qr(int64_t m, int64_t w, double* P, int64_t ldp, double* tau) {
  int64_t kk = m < w ? m : w;
  for (int64_t t = 0; t < kk; ++t) {
    double beta;
    double tt = oracle_house(m - t, &AT(P, t, t, ldp), 1, &beta);
    tau[t] = tt;
    if (tt != 0.0) {
      for (int64_t j = t + 1; j < w; ++j) {
        double s = AT(P, t, j, ldp);
        for (int64_t r = t + 1; r < m; ++r) s += AT(P, r, t, ldp) * AT(P, r, j, ldp);
        s *= tt;
        AT(P, t, j, ldp) -= s;
        for (int64_t r = t + 1; r < m; ++r) AT(P, r, j, ldp) -= s * AT(P, r, t, ldp);
      }
    }
    AT(P, t, t, ldp) = beta;
  }
}

/* Reflector t as a dense column: v[r] = 0 (r < t), 1 (r == t), V(r,t) (r > t). */
static void unit_col(int64_t m, int64_t t, const double* V, int64_t ldv, double* v) {
  for (int64_t r = 0; r < m; ++r) v[r] = r < t ? 0.0 : (r == t ? 1.0 : AT(V, r, t, ldv));
}

/* H_{k+1} = I - w y^T with y = v, w = tau v;  W_{k+1} = [W_k | w - W_k Y_k^T w]. */
void oracle_wy(int64_t m, int64_t kk, const double* V, int64_t ldv, const double* tau, double* W, int64_t ldw) {
  double* y = zalloc((size_t)m);
  double* w = zalloc((size_t)m);
  double* yk = zalloc((size_t)m);
  for (int64_t t = 0; t < kk; ++t) {
    unit_col(m, t, V, ldv, y);
    for (int64_t r = 0; r < m; ++r) w[r] = tau[t] * y[r];
    for (int64_t q = 0; q < t; ++q) {        /* w -= W_k (Y_k^T w) */
      unit_col(m, q, V, ldv, yk);
      double s = 0.0;
      for (int64_t r = 0; r < m; ++r) s += yk[r] * (tau[t] * y[r]);
      for (int64_t r = 0; r < m; ++r) w[r] -= AT(W, r, q, ldw) * s;
    }
    for (int64_t r = 0; r < m; ++r) AT(W, r, t, ldw) = w[r];
  }
  free(y); free(w); free(yk);
}

/* Eq. (1): Z = A W - 1/2 Y W^T A W. */
void oracle_zy(int64_t m, int64_t kk, const double* A, int64_t lda, const double* W, int64_t ldw,
               const double* Y, int64_t ldy, double* Z, int64_t ldz) {
  double* X = zalloc((size_t)(m * kk));   /* X = A W */
  double* S = zalloc((size_t)(kk * kk));  /* S = W^T X */
  for (int64_t c = 0; c < kk; ++c)
    for (int64_t i = 0; i < m; ++i) {
      double s = 0.0;
      for (int64_t j = 0; j < m; ++j) s += sym_get(A, lda, i, j) * AT(W, j, c, ldw);
      X[c * m + i] = s;
    }
  for (int64_t c = 0; c < kk; ++c)
    for (int64_t r = 0; r < kk; ++r) {
      double s = 0.0;
      for (int64_t i = 0; i < m; ++i) s += AT(W, i, r, ldw) * X[c * m + i];
      S[c * kk + r] = s;
    }
  for (int64_t c = 0; c < kk; ++c)
    for (int64_t i = 0; i < m; ++i) {
      double s = 0.0;
      for (int64_t r = 0; r < kk; ++r) s += AT(Y, i, r, ldy) * S[c * kk + r];
      AT(Z, i, c, ldz) = X[c * m + i] - 0.5 * s;
    }
  free(X); free(S);
}

/* syr2k lower (Alg. 1 l.15): C(i,j) -= sum_l Y(i,l) Z(j,l) + Z(i,l) Y(j,l), i >= j. */
void oracle_syr2k_lower(int64_t m, int64_t kk, double* C, int64_t ldc, const double* Y, int64_t ldy,
                        const double* Z, int64_t ldz) {
  for (int64_t j = 0; j < m; ++j)
    for (int64_t i = j; i < m; ++i) {
      double s = 0.0;
      for (int64_t l = 0; l < kk; ++l) s += AT(Y, i, l, ldy) * AT(Z, j, l, ldz) + AT(Z, i, l, ldz) * AT(Y, j, l, ldy);
      AT(C, i, j, ldc) -= s;
    }
}

/* Algorithm 1, readings R4(a)-(f). */
void oracle_dbbr(int64_t n, int64_t b, int64_t k, double* A, int64_t lda, double* tau1) {
  for (int64_t c = 0; c < n; ++c) tau1[c] = 0.0;
  if (n <= 0 || b < 1 || k < b) return;
  int64_t kcols = k;
  double* Y = zalloc((size_t)(n * kcols));  /* global row index; block columns */
  double* Z = zalloc((size_t)(n * kcols));
  for (int64_t i = 0; i + b + 1 < n; i += k) {                          /* l.1 (R4f: stop at n-b-1) */
    memset(Y, 0, sizeof(double) * (size_t)(n * kcols));
    memset(Z, 0, sizeof(double) * (size_t)(n * kcols));                 /* R4c: reset per block */
    int64_t ncols = 0, j_last = i;
    for (int64_t j = i; j < i + k && j + b + 1 < n; j += b) {          /* l.3 (R4b) */
      int64_t o = j + b, m = n - o, w = b, kk = m < w ? m : w;
      /* l.5: PanelQR(A(j+b:n, j:j+b)) -> y (= V) and z */
      double* tau = zalloc((size_t)w);
      oracle_panel_qr(m, w, &AT(A, o, j, lda), lda, tau);
      for (int64_t t = 0; t < kk; ++t) tau1[j + t] = tau[t];
      double* W = zalloc((size_t)(m * kk));
      oracle_wy(m, kk, &AT(A, o, j, lda), lda, tau, W, m);
      /* implicitly updated trailing matrix A_cur = A(o:, o:) - Yprev Zprev^T - Zprev Yprev^T (R4e) */
      double* Acur = zalloc((size_t)(m * m));
      for (int64_t c = 0; c < m; ++c)
        for (int64_t r = c; r < m; ++r) {
          double s = AT(A, o + r, o + c, lda);
          for (int64_t l = 0; l < ncols; ++l)
            s -= Y[l * n + o + r] * Z[l * n + o + c] + Z[l * n + o + r] * Y[l * n + o + c];
          Acur[c * m + r] = s;
        }
      double* Yp = zalloc((size_t)(m * kk));
      for (int64_t t = 0; t < kk; ++t) unit_col(m, t, &AT(A, o, j, lda), lda, &Yp[t * m]);
      double* Zp = zalloc((size_t)(m * kk));
      oracle_zy(m, kk, Acur, m, W, m, Yp, m, Zp, m);                     /* Eq. (1) */
      for (int64_t t = 0; t < kk; ++t)                                   /* l.6: Z = [Z|z]; Y = [Y|y] */
        for (int64_t r = 0; r < m; ++r) {
          Y[(ncols + t) * n + o + r] = Yp[t * m + r];
          Z[(ncols + t) * n + o + r] = Zp[t * m + r];
        }
      ncols += kk;
      j_last = j;
      int64_t jn = j + b;
      int last = !(jn < i + k && jn + b + 1 < n);
      if (!last) {                                                       /* l.8-12 (R4d: skip for last) */
        for (int64_t c = o; c < o + b && c < n; ++c)
          for (int64_t r = c; r < n; ++r) {                               /* lower part only (R6) */
            double s = 0.0;
            for (int64_t l = 0; l < ncols; ++l) s += Z[l * n + r] * Y[l * n + c] + Y[l * n + r] * Z[l * n + c];
            AT(A, r, c, lda) -= s;
          }
      }
      free(tau); free(W); free(Acur); free(Yp); free(Zp);
    }
    /* l.15: A(e:n, e:n) = syr2k(A(e:n, e:n), Z, Y) with e = end of the block's last panel */
    int64_t e = j_last + b;
    if (e < n) oracle_syr2k_lower(n - e, ncols, &AT(A, e, e, lda), lda, &Y[e], n, &Z[e], n);
  }
  free(Y); free(Z);
}

/* Reading R7: step m of sweep s exists iff s+1+m*b <= n-2. */
int64_t oracle_bc_steps(int64_t n, int64_t b, int64_t s) {
  if (b < 2 || s < 0 || s > n - 3) return 0;
  return (n - 3 - s) / b + 1;
}

int64_t oracle_bc_total_steps(int64_t n, int64_t b) {
  int64_t t = 0;
  for (int64_t s = 0; s + 3 <= n; ++s) t += oracle_bc_steps(n, b, s);
  return t;
}

/* One bulge-chasing step (s, m) on the dense full-storage copy M (n x n, ld n) (sec. 2.4, Fig. 3, Alg. 2;
 * step indexing R7).  H from column col (= s for m = 0, else the first column of the previous block, which
 * holds the bulge's first column) over rows R_m = [r0, r1]; then M <- H M H, i.e. left-apply to the
 * off-band block (B_ol), two-sided to the diagonal block (B_d), right-apply to the block below (B_od,
 * which creates the bulge).  The eliminated entries are set to beta / exact zero.  full != 0 applies H to
 * the whole matrix instead of the window rows/columns r0-2b .. r1+2b.  v (b doubles) and tmp (n) are
 * scratch; the reflector goes to V2[off*b ..] / tau2[off] when those are non-NULL. */
static void bc_step(int64_t n, int64_t b, double* M, int64_t s, int64_t m, int64_t off, double* V2, double* tau2,
                    int full, double* v, double* tmp) {
  int64_t r0 = s + 1 + m * b;
  int64_t r1 = s + (m + 1) * b; if (r1 > n - 1) r1 = n - 1;
  int64_t L = r1 - r0 + 1;
  int64_t col = (m == 0) ? s : r0 - b;
  for (int64_t r = 0; r < L; ++r) v[r] = M[col * n + r0 + r];
  double beta;
  double tau = oracle_house(L, v, 1, &beta);
  v[0] = 1.0;
  if (V2) { for (int64_t r = 0; r < b; ++r) V2[off * b + r] = r < L ? v[r] : 0.0; }
  if (tau2) tau2[off] = tau;
  if (tau != 0.0) {
    int64_t lo = full ? 0 : (r0 - 2 * b > 0 ? r0 - 2 * b : 0);
    int64_t hi = full ? n - 1 : (r1 + 2 * b < n - 1 ? r1 + 2 * b : n - 1);
    /* left: rows R_m of columns lo..hi */
    for (int64_t c = lo; c <= hi; ++c) {
      double sum = 0.0;
      for (int64_t r = 0; r < L; ++r) sum += v[r] * M[c * n + r0 + r];
      sum *= tau;
      for (int64_t r = 0; r < L; ++r) M[c * n + r0 + r] -= sum * v[r];
    }
    /* right: columns R_m of rows lo..hi */
    for (int64_t i = lo; i <= hi; ++i) {
      double sum = 0.0;
      for (int64_t r = 0; r < L; ++r) sum += M[(r0 + r) * n + i] * v[r];
      tmp[i] = tau * sum;
    }
    for (int64_t r = 0; r < L; ++r)
      for (int64_t i = lo; i <= hi; ++i) M[(r0 + r) * n + i] -= tmp[i] * v[r];
  }
  M[col * n + r0] = beta; M[r0 * n + col] = beta;
  for (int64_t r = 1; r < L; ++r) { M[col * n + r0 + r] = 0.0; M[(r0 + r) * n + col] = 0.0; }
}

/* Dense full-storage copy of the band (diagonal + b subdiagonals of A's lower triangle). */
static double* bc_dense_band(int64_t n, int64_t b, const double* A, int64_t lda) {
  double* M = zalloc((size_t)(n * n));
  for (int64_t j = 0; j < n; ++j)
    for (int64_t i = j; i < n && i <= j + b; ++i) { M[j * n + i] = AT(A, i, j, lda); M[i * n + j] = AT(A, i, j, lda); }
  return M;
}

static void bc_extract(int64_t n, const double* M, double* d, double* e) {
  for (int64_t i = 0; i < n; ++i) d[i] = M[i * n + i];
  for (int64_t i = 0; i + 1 < n; ++i) e[i] = M[i * n + i + 1];
}

/* O2b: naive sweep-major bulge chasing (sec. 2.4, Fig. 3, Alg. 2). */
void oracle_bc_naive(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e,
                     double* V2, double* tau2, int full) {
  if (n <= 0) return;
  double* M = bc_dense_band(n, b, A, lda);
  double* v = zalloc((size_t)(b > 1 ? b : 1));
  double* tmp = zalloc((size_t)n);
  int64_t off = 0;
  if (b >= 2) {
    for (int64_t s = 0; s + 3 <= n; ++s) {
      int64_t nst = oracle_bc_steps(n, b, s);
      for (int64_t m = 0; m < nst; ++m, ++off) bc_step(n, b, M, s, m, off, V2, tau2, full, v, tmp);
    }
  }
  bc_extract(n, M, d, e);
  free(M); free(v); free(tmp);
}

/* The paper's pipelined order (reading R9) executed serially: in time slot t every
 * sweep s with 0 <= t - lag*s < steps(s) runs its step m = t - lag*s, the sweeps of one slot taken from the
 * highest s down (the order in which a real pipeline may complete them: a later sweep never waits for an
 * earlier sweep's step of the same slot).  lag >= 1.  With lag >= 2 no step reads a window another step of
 * its slot writes, so the result is the sweep-major one bit for bit; lag 1 lets sweep s read sweep s-1's
 * window before sweep s-1 has updated it. */
void oracle_bc_wavefront(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e,
                         double* V2, double* tau2, int64_t lag) {
  if (n <= 0) return;
  double* M = bc_dense_band(n, b, A, lda);
  double* v = zalloc((size_t)(b > 1 ? b : 1));
  double* tmp = zalloc((size_t)n);
  if (b >= 2 && n >= 3 && lag >= 1) {
    const int64_t ns = n - 2;
    int64_t* S = (int64_t*)calloc((size_t)ns + 1, sizeof(int64_t));
    if (!S) abort();
    for (int64_t s = 0; s < ns; ++s) S[s + 1] = S[s] + oracle_bc_steps(n, b, s);
    const int64_t tmax = lag * (ns - 1) + oracle_bc_steps(n, b, 0);
    for (int64_t t = 0; t < tmax; ++t) {
      for (int64_t s = ns - 1; s >= 0; --s) {
        const int64_t m = t - lag * s;
        if (m < 0 || m >= oracle_bc_steps(n, b, s)) continue;
        bc_step(n, b, M, s, m, S[s] + m, V2, tau2, 0, v, tmp);
      }
    }
    free(S);
  }
  bc_extract(n, M, d, e);
  free(M); free(v); free(tmp);
}

/* O2c: the same chase with the step grouping of reading R7, on the lower triangle only: step (s, m) owns the
 * columns R_m.  Given its reflector v (generated from column s at m = 0, else by step m-1 of the sweep) it
 * applies H = I - tau v v^T two-sided to D = B(R_m, R_m) (p = tau D v, w = p - 1/2 tau (p^T v) v,
 * D -= v w^T + w v^T), from the right to O = B(R_{m+1}, R_m) (O -= tau (O v) v^T), generates the next
 * reflector from O(:, 0) and applies it from the left to O(:, 1:) (the paper's "left-apply to B_ol" of the
 * next step, moved into this one).  Same reflectors and T as O2b up to rounding.
 * lag = 0: sweep-major order.  lag >= 1: the wavefront order of oracle_bc_wavefront (slot t runs step
 * t - lag*s of every sweep, highest s first).  With this grouping a step touches only its own columns R_m
 * (rows R_m u R_{m+1}), so lag 2 is the minimal lag that reproduces the sweep-major result bit for bit
 * (reading R9); lag 1 reads a window before its predecessor finished it. */
void oracle_bc_r7(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e, double* V2,
                  double* tau2, int64_t lag) {
  if (n <= 0) return;
  double* M = zalloc((size_t)(n * n));   /* lower triangle only: M(i, j) = M[j*n + i], i >= j */
  for (int64_t j = 0; j < n; ++j)
    for (int64_t i = j; i < n && i <= j + b; ++i) M[j * n + i] = AT(A, i, j, lda);
  if (b >= 2 && n >= 3) {
    const int64_t ns = n - 2;
    int64_t* S = (int64_t*)calloc((size_t)ns + 1, sizeof(int64_t));
    double* vpend = zalloc((size_t)(ns * b));   /* per sweep: the reflector of its next step */
    double* tpend = zalloc((size_t)ns);
    double* p = zalloc((size_t)b);
    double* y = zalloc((size_t)b);
    double* z = zalloc((size_t)b);
    if (!S) abort();
    for (int64_t s = 0; s < ns; ++s) S[s + 1] = S[s] + oracle_bc_steps(n, b, s);
    const int64_t lg = lag >= 1 ? lag : 0;
    const int64_t tmax = lg ? lg * (ns - 1) + oracle_bc_steps(n, b, 0) : 1;
    for (int64_t t = 0; t < tmax; ++t) {
      for (int64_t q = 0; q < ns; ++q) {
        const int64_t s = lg ? ns - 1 - q : q;
        const int64_t m0 = lg ? t - lg * s : 0, m1 = lg ? m0 + 1 : oracle_bc_steps(n, b, s);
        if (lg && (m0 < 0 || m0 >= oracle_bc_steps(n, b, s))) continue;
        for (int64_t m = m0; m < m1; ++m) {
          double* v = &vpend[s * b];
          const int64_t r0 = s + 1 + m * b;
          int64_t r1 = s + (m + 1) * b; if (r1 > n - 1) r1 = n - 1;
          const int64_t L = r1 - r0 + 1;
          int64_t r2 = r1 + b; if (r2 > n - 1) r2 = n - 1;
          const int64_t L2 = r2 - r1;
          double tau;
          if (m == 0) {   /* the reflector annihilating column s below its first subdiagonal */
            for (int64_t r = 0; r < L; ++r) v[r] = M[s * n + r0 + r];
            double beta;
            tau = oracle_house(L, v, 1, &beta);
            v[0] = 1.0;
            M[s * n + r0] = beta;
            for (int64_t r = 1; r < L; ++r) M[s * n + r0 + r] = 0.0;
          } else {
            tau = tpend[s];
          }
          if (V2) for (int64_t r = 0; r < b; ++r) V2[(S[s] + m) * b + r] = r < L ? v[r] : 0.0;
          if (tau2) tau2[S[s] + m] = tau;
          if (tau != 0.0) {
            /* two-sided on D (lower), right-apply to O */
            for (int64_t i = 0; i < L; ++i) {
              double acc = 0.0;
              for (int64_t j = 0; j < L; ++j) {
                const int64_t gi = r0 + i, gj = r0 + j;
                acc += (gi >= gj ? M[gj * n + gi] : M[gi * n + gj]) * v[j];
              }
              p[i] = tau * acc;
            }
            for (int64_t i = 0; i < L2; ++i) {
              double acc = 0.0;
              for (int64_t j = 0; j < L; ++j) acc += M[(r0 + j) * n + r1 + 1 + i] * v[j];
              y[i] = acc;
            }
            double pv = 0.0;
            for (int64_t i = 0; i < L; ++i) pv += p[i] * v[i];
            const double hp = 0.5 * tau * pv;
            for (int64_t i = 0; i < L; ++i) p[i] -= hp * v[i];   /* p is now w */
            for (int64_t j = 0; j < L; ++j)
              for (int64_t i = j; i < L; ++i) M[(r0 + j) * n + r0 + i] -= v[i] * p[j] + p[i] * v[j];
            for (int64_t j = 0; j < L; ++j)
              for (int64_t i = 0; i < L2; ++i) M[(r0 + j) * n + r1 + 1 + i] -= tau * y[i] * v[j];
          }
          if (L2 > 0) {   /* next reflector from O(:, 0), left-applied to O(:, 1:) */
            double* vn = z;   /* reuse: vn then copied into vpend */
            for (int64_t i = 0; i < L2; ++i) vn[i] = M[r0 * n + r1 + 1 + i];
            double beta;
            const double tn = oracle_house(L2, vn, 1, &beta);
            vn[0] = 1.0;
            M[r0 * n + r1 + 1] = beta;
            for (int64_t i = 1; i < L2; ++i) M[r0 * n + r1 + 1 + i] = 0.0;
            if (tn != 0.0) {
              for (int64_t j = 1; j < L; ++j) {
                double acc = 0.0;
                for (int64_t i = 0; i < L2; ++i) acc += vn[i] * M[(r0 + j) * n + r1 + 1 + i];
                acc *= tn;
                for (int64_t i = 0; i < L2; ++i) M[(r0 + j) * n + r1 + 1 + i] -= acc * vn[i];
              }
            }
            for (int64_t i = 0; i < b; ++i) v[i] = i < L2 ? vn[i] : 0.0;
            tpend[s] = tn;
          }
        }
      }
    }
    free(S); free(vpend); free(tpend); free(p); free(y); free(z);
  }
  for (int64_t i = 0; i < n; ++i) d[i] = M[i * n + i];
  for (int64_t i = 0; i + 1 < n; ++i) e[i] = M[i * n + i + 1];
  free(M);
}

/* Q = Q1 Q2 (reading R2).  Right-multiplying by H = I - tau v v^T on index range [o, o+L). */
static void q_right_apply(int64_t n, double* Q, int64_t ldq, int64_t o, int64_t L, const double* v, double tau) {
  if (tau == 0.0) return;
  for (int64_t i = 0; i < n; ++i) {
    double s = 0.0;
    for (int64_t r = 0; r < L; ++r) s += AT(Q, i, o + r, ldq) * v[r];
    s *= tau;
    for (int64_t r = 0; r < L; ++r) AT(Q, i, o + r, ldq) -= s * v[r];
  }
}

void oracle_form_q(int64_t n, int64_t b, const double* A_sbr, int64_t lda, const double* tau1,
                   const double* V2, const double* tau2, double* Q, int64_t ldq) {
  for (int64_t j = 0; j < n; ++j)
    for (int64_t i = 0; i < n; ++i) AT(Q, i, j, ldq) = (i == j) ? 1.0 : 0.0;
  double* v = zalloc((size_t)n);
  if (tau1 && A_sbr) {
    for (int64_t c = 0; c + b + 1 < n; ++c) {
      int64_t o = c + b, L = n - o;
      v[0] = 1.0;
      for (int64_t r = 1; r < L; ++r) v[r] = AT(A_sbr, o + r, c, lda);
      q_right_apply(n, Q, ldq, o, L, v, tau1[c]);
    }
  }
  if (V2 && tau2 && b >= 2) {
    int64_t off = 0;
    for (int64_t s = 0; s + 3 <= n; ++s) {
      int64_t nst = oracle_bc_steps(n, b, s);
      for (int64_t m = 0; m < nst; ++m, ++off) {
        int64_t r0 = s + 1 + m * b;
        int64_t r1 = s + (m + 1) * b; if (r1 > n - 1) r1 = n - 1;
        q_right_apply(n, Q, ldq, r0, r1 - r0 + 1, &V2[off * b], tau2[off]);
      }
    }
  }
  free(v);
}

/* SBR back-transformation (sec. 4.3): C <- Q1 C (trans = 0) or Q1^T C
 * (trans = 1), Q1 = H_0 H_1 ... H_{n-b-2} with H_c = I - tau1[c] v_c v_c^T, v_c = (1, A(c+b+1:n-1, c)) on rows
 * c+b..n-1 (the layout trid_sbr_dbbr leaves).  The definition, one reflector at a time: Q1 C applies H_{n-b-2}
 * first, Q1^T C applies H_0 first.  (The paper's Alg. 3 merges the W blocks into wider ones; that regrouping is
 * the method, this is the result it must reach.)  C is n x ncols, column-major, ld ldc. */
void oracle_sbr_backtransform(int64_t n, int64_t b, const double* A, int64_t lda, const double* tau1, int trans,
                              int64_t ncols, double* C, int64_t ldc) {
  if (n <= 0 || ncols <= 0) return;
  double* v = zalloc((size_t)n);
  const int64_t last = n - b - 2;
  for (int64_t q = 0; q <= last; ++q) {
    const int64_t c = trans ? q : last - q;
    const double tau = tau1[c];
    if (tau == 0.0) continue;
    const int64_t o = c + b, L = n - o;
    v[0] = 1.0;
    for (int64_t r = 1; r < L; ++r) v[r] = AT(A, o + r, c, lda);
    for (int64_t j = 0; j < ncols; ++j) {
      double s = 0.0;
      for (int64_t r = 0; r < L; ++r) s += v[r] * AT(C, o + r, j, ldc);
      s *= tau;
      for (int64_t r = 0; r < L; ++r) AT(C, o + r, j, ldc) -= s * v[r];
    }
  }
  free(v);
}

/* BC back-transformation: C <- Q2 C (trans = 0) or Q2^T C (trans = 1),
 * Q2 = prod over sweeps s (ascending) and steps m (ascending) of H_{s,m} = I - tau2 v v^T (the R7 layout of
 * trid_bulge_chase: v at V2[(S(s)+m)*b], rows s+1+m*b .. min(s+(m+1)*b, n-1)).  The definition, one
 * reflector at a time: Q2 C applies the last reflector first. */
void oracle_bc_backtransform(int64_t n, int64_t b, const double* V2, const double* tau2, int trans, int64_t ncols,
                             double* C, int64_t ldc) {
  if (n < 3 || b < 2 || ncols <= 0) return;
  const int64_t tot = oracle_bc_total_steps(n, b);
  int64_t* sw = (int64_t*)calloc((size_t)tot, sizeof(int64_t));
  int64_t* st = (int64_t*)calloc((size_t)tot, sizeof(int64_t));
  if (!sw || !st) abort();
  int64_t off = 0;
  for (int64_t s = 0; s + 3 <= n; ++s)
    for (int64_t m = 0; m < oracle_bc_steps(n, b, s); ++m, ++off) { sw[off] = s; st[off] = m; }
  for (int64_t q = 0; q < tot; ++q) {
    const int64_t i = trans ? q : tot - 1 - q;
    const double tau = tau2[i];
    if (tau == 0.0) continue;
    const int64_t r0 = sw[i] + 1 + st[i] * b;
    int64_t r1 = sw[i] + (st[i] + 1) * b; if (r1 > n - 1) r1 = n - 1;
    const int64_t L = r1 - r0 + 1;
    const double* v = &V2[i * b];
    for (int64_t j = 0; j < ncols; ++j) {
      double s = 0.0;
      for (int64_t r = 0; r < L; ++r) s += v[r] * AT(C, r0 + r, j, ldc);
      s *= tau;
      for (int64_t r = 0; r < L; ++r) AT(C, r0 + r, j, ldc) -= s * v[r];
    }
  }
  free(sw); free(st);
}

/* Sturm count: number of eigenvalues < x (LAPACK dlaebz-style pivot guard). */
int64_t oracle_sturm_count(int64_t n, const double* d, const double* e, double x, double pivmin) {
  int64_t cnt = 0;
  double q = d[0] - x;
  if (fabs(q) < pivmin) q = -pivmin;
  if (q < 0) ++cnt;
  for (int64_t i = 1; i < n; ++i) {
    q = d[i] - x - e[i - 1] * e[i - 1] / q;
    if (fabs(q) < pivmin) q = -pivmin;
    if (q < 0) ++cnt;
  }
  return cnt;
}

void oracle_sturm_eig(int64_t n, const double* d, const double* e, double* w) {
  if (n <= 0) return;
  double gl = d[0], gu = d[0], emax2 = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    double r = (i > 0 ? fabs(e[i - 1]) : 0.0) + (i + 1 < n ? fabs(e[i]) : 0.0);
    if (d[i] - r < gl) gl = d[i] - r;
    if (d[i] + r > gu) gu = d[i] + r;
    if (i + 1 < n && e[i] * e[i] > emax2) emax2 = e[i] * e[i];
  }
  double pivmin = DBL_MIN * (emax2 > 1.0 ? emax2 : 1.0);
  double span = gu - gl, scale = fabs(gl) > fabs(gu) ? fabs(gl) : fabs(gu);
  gl -= 2.0 * DBL_EPSILON * scale + 2.0 * pivmin + 1e-300 + 0.0 * span;
  gu += 2.0 * DBL_EPSILON * scale + 2.0 * pivmin + 1e-300;
  for (int64_t k = 0; k < n; ++k) {
    double lo = gl, hi = gu;
    for (int it = 0; it < 256; ++it) {
      double tol = 2.0 * DBL_EPSILON * (fabs(lo) > fabs(hi) ? fabs(lo) : fabs(hi)) + pivmin;
      if (hi - lo <= tol) break;
      double mid = 0.5 * (lo + hi);
      if (mid <= lo || mid >= hi) break;
      if (oracle_sturm_count(n, d, e, mid, pivmin) > k) hi = mid; else lo = mid;
    }
    w[k] = 0.5 * (lo + hi);
  }
}

/* Cyclic-by-row Jacobi (Golub & Van Loan, Alg. 8.5.2/8.5.3). */
static int dcmp(const void* a, const void* b) {
  double x = *(const double*)a, y = *(const double*)b;
  return x < y ? -1 : (x > y ? 1 : 0);
}

int oracle_jacobi_eig(int64_t n, double* A, int64_t lda, double* w) {
  double fro = 0.0;
  for (int64_t j = 0; j < n; ++j)
    for (int64_t i = 0; i < n; ++i) fro += AT(A, i, j, lda) * AT(A, i, j, lda);
  fro = sqrt(fro);
  int sweeps = 0;
  for (; sweeps < 100; ++sweeps) {
    double off = 0.0;
    for (int64_t j = 0; j < n; ++j)
      for (int64_t i = 0; i < n; ++i)
        if (i != j) off += AT(A, i, j, lda) * AT(A, i, j, lda);
    if (sqrt(off) <= 1e-15 * fro) break;
    for (int64_t p = 0; p < n - 1; ++p)
      for (int64_t q = p + 1; q < n; ++q) {
        double apq = AT(A, p, q, lda);
        if (apq == 0.0) continue;
        double app = AT(A, p, p, lda), aqq = AT(A, q, q, lda);
        double theta = (aqq - app) / (2.0 * apq);
        double t = (theta >= 0 ? 1.0 : -1.0) / (fabs(theta) + sqrt(1.0 + theta * theta));
        double c = 1.0 / sqrt(1.0 + t * t), s = t * c;
        for (int64_t k = 0; k < n; ++k) {   /* A = A J */
          double akp = AT(A, k, p, lda), akq = AT(A, k, q, lda);
          AT(A, k, p, lda) = c * akp - s * akq;
          AT(A, k, q, lda) = s * akp + c * akq;
        }
        for (int64_t k = 0; k < n; ++k) {   /* A = J^T A */
          double apk = AT(A, p, k, lda), aqk = AT(A, q, k, lda);
          AT(A, p, k, lda) = c * apk - s * aqk;
          AT(A, q, k, lda) = s * apk + c * aqk;
        }
      }
  }
  for (int64_t i = 0; i < n; ++i) w[i] = AT(A, i, i, lda);
  qsort(w, (size_t)n, sizeof(double), dcmp);
  return sweeps;
}
