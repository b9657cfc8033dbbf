// api.cu — the C-ABI of libtrid.so (include/trid.h): argument checks, workspace carving and the
// host-side DBBR driver (Alg. 1, with readings R4a-f), all stream-ordered.
//
// Per panel p at column j of the outer block starting at i (m = n-j-b trailing rows, kk = min(b, m)):
//   a1/a2  panel_qr     : V (in A), tau1, T, explicit Y_p                         (Alg. 1 l.5)
//          W_p = Y_p T   (DMMA)
//   a3     X = A_blk(j+b:, j+b:) W_p  (SYMM on the block-start trailing matrix, lower-stored)
//          X -= Y_<p (Z_<p^T W_p) + Z_<p (Y_<p^T W_p)   (implicit update by earlier panels, R4e)
//          Z_p = X - 1/2 Y_p (W_p^T X)                                              (Eq. (1))
//   a4     next-panel update A(j+b:, j+b:j+2b) -= Z Y^T + Y Z^T (all but the block's last panel, R4d)
// and per block:
//   a5     syr2k  A(e:, e:) -= Y Z^T + Z Y^T  lower triangle, e = end of the block's last panel (l.15)
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <atomic>
#include <mutex>
#include <vector>

#include "../../include/trid.h"
#include "common.cuh"
#include "gemm.cuh"
#include "panel.cuh"
#include "prof.cuh"
#include "driver.cuh"
#include "eig.cuh"
#include "backtrans.cuh"

using namespace trid;

namespace {

// ---- optional stage profiling (trid_profile_*) and launch counting ------------------------------
std::atomic<long long> g_launches{0};
struct ProfState {
  std::mutex mu;
  bool on = false;
  std::vector<cudaEvent_t> pool;
  size_t used = 0;
  cudaEvent_t open[PROF_NCLASS] = {};
  std::vector<cudaEvent_t> begins[PROF_NCLASS], ends[PROF_NCLASS];
};
ProfState& prof() {
  static ProfState p;
  return p;
}
cudaEvent_t prof_event(ProfState& p) {
  if (p.used == p.pool.size()) {
    cudaEvent_t ev;
    if (cudaEventCreate(&ev) != cudaSuccess) return nullptr;
    p.pool.push_back(ev);
  }
  return p.pool[p.used++];
}

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

struct Carver {
  char* base;
  size_t off = 0;
  explicit Carver(void* p) : base((char*)p) {}
  template <class T>
  T* take(size_t count) {
    T* p = base ? (T*)(base + off) : nullptr;
    off += align256(sizeof(T) * count);
    return p;
  }
};

int default_k(int64_t n, int b) {
  (void)n;
  int cap = b > 1024 ? b : 1024;
  return (cap / b) * b;
}

// largest SYMM split-K partial footprint over all panels of the reduction
int64_t max_symm_part(int64_t n, int b, int k) {
  int64_t best = 0;
  for (int64_t j = 0; j + b + 1 < n; j += b) {
    const int64_t m = n - j - b;
    const int64_t kk = m < b ? m : b;
    int64_t e = symm_ws_part_elems(m, kk);
    const int64_t ef = symm_ws_part_elems(m, kk, j % k);   // with the block's corrections folded in
    if (ef > e) e = ef;
    if (e > best) best = e;
  }
  return best;
}

// split-K partial footprint bound of the skinny engine GEMMs (M = m <= n - b, N = b, <= 16 splits)
int64_t max_skinny_part(int64_t n, int b, int k) {
  (void)k;
  const int64_t m = n - b > 0 ? n - b : 0;
  return (int64_t)16 * m * b;
}

struct DbbrWork {
  double *Y, *Z, *W, *X, *T, *U, *S, *part, *red;
  unsigned *bar, *sem;
  int64_t part_elems;
  size_t bytes;
};

DbbrWork carve_dbbr(void* base, int64_t n, int b, int k) {
  DbbrWork w;
  Carver c(base);
  w.Y = c.take<double>((size_t)n * k);
  w.Z = c.take<double>((size_t)n * k);
  w.W = c.take<double>((size_t)n * b);
  w.X = c.take<double>((size_t)n * b);
  w.T = c.take<double>((size_t)b * b);
  w.U = c.take<double>((size_t)2 * k * b);   // [Z_<^T W; Y_<^T W], ld 2k
  w.S = c.take<double>((size_t)b * b);
  int64_t pe = max_symm_part(n, b, k);
  const int64_t tn = (int64_t)64 * k * b;  // split-K partials of the tall reductions (2k x b stacked)
  if (pe < tn) pe = tn;
  const int64_t sk = max_skinny_part(n, b, k);   // next-panel update / corrections split-K
  if (pe < sk) pe = sk;
  w.part_elems = pe;
  w.part = c.take<double>((size_t)pe);
  w.red = (double*)c.take<char>(panel_red_bytes(b));
  w.bar = c.take<unsigned>(256);   // panel grid-barrier counters (8 x 128 B)
  w.sem = c.take<unsigned>(1024);
  w.bytes = c.off;
  return w;
}

}  // namespace

namespace trid {
// C = alpha A B + beta Cin with a short inner dimension (K <= b: W = Y T, Z = X - 1/2 Y S).  Measured at
// n = 32768 (gpurun_out/r01x/env): the persistent warp-specialized engine beats the plain multi-CTA engine
// here (wy 11.4 vs 14.6 ms, zy 142 vs 147 ms per step), so it is the default; TRID_SKINNY_WS=0 selects the
// plain engine (A/B).
cudaError_t gemm_skinny_k(GemmArgs g, cudaStream_t st) {
  static const bool plain = getenv("TRID_SKINNY_WS") != nullptr && getenv("TRID_SKINNY_WS")[0] == '0';
  if (!plain) return gemm_ws(g, OP_N, st);
  g.splits = 1;
  return gemm(g, OP_N, OP_N, TILE_128x64, st);
}

// ---- the Z builder after the SYMM (a3): corrections for the block's earlier panels (R4e), S = W^T X,
// Z_p = X - 1/2 Y_p S (Eq. (1)).  X (m x kk, ld ldx) holds A_blk W_p on entry and is updated.
// folded: the corrections were already applied inside the SYMM launch (zy_panel), only S and Z remain.
cudaError_t zy_tail(int64_t m, int kk, const double* Wp, int64_t ldw, const double* Yp, const double* Yprev,
                    const double* Zprev, int64_t ldyz, int64_t nprev, double* Zp, double* X, int64_t ldx, double* U,
                    int64_t ldu, double* S, int64_t lds, double* part, int64_t part_elems, unsigned* sem,
                    cudaStream_t st, bool folded) {
  cudaError_t e;
  ProfScope ps(PROF_ZY, st);
  if (nprev > 0 && !folded) {
    // [U1; U2] = [Z_<^T W; Y_<^T W]   (TN, K = m, deterministic split-K; one launch, stacked rows)
    double* U1 = U;
    double* U2 = U + nprev;
    GemmArgs g;
    g.M = 2 * nprev; g.N = kk; g.K[0] = m; g.A[0] = Zprev; g.lda[0] = ldyz; g.B[0] = Wp; g.ldb[0] = ldw;
    g.A2m = Yprev; g.msplit = nprev;
    g.C = U; g.ldc = ldu; g.alpha = 1.0; g.beta = 0.0;
    g.splits = pick_splits(2 * nprev, kk, m, TILE_64x64, part_elems);
    g.part = part; g.part_ld = 2 * nprev; g.part_stride = 2 * nprev * kk;
    static const bool u_ws = !(getenv("TRID_ZY_WS") && getenv("TRID_ZY_WS")[0] == '0');
    if (u_ws) {
      // the two stacked TN products on the warp-specialized engine (op(A) = A^T), one launch per operand
      if ((e = gemm_ws_mm(OP_T, OP_N, nprev, kk, m, 1.0, Zprev, ldyz, Wp, ldw, 0.0, U1, ldu, part, part_elems, st)) !=
          cudaSuccess)
        return e;
      if ((e = gemm_ws_mm(OP_T, OP_N, nprev, kk, m, 1.0, Yprev, ldyz, Wp, ldw, 0.0, U2, ldu, part, part_elems, st)) !=
          cudaSuccess)
        return e;
    } else if ((e = gemm(g, OP_T, OP_N, TILE_64x64, st)) != cudaSuccess) {
      return e;
    }
    // X -= Y_< U1 + Z_< U2
    GemmArgs h;
    h.M = m; h.N = kk; h.nseg = 2;
    h.A[0] = Yprev; h.lda[0] = ldyz; h.B[0] = U1; h.ldb[0] = ldu; h.K[0] = nprev;
    h.A[1] = Zprev; h.lda[1] = ldyz; h.B[1] = U2; h.ldb[1] = ldu; h.K[1] = nprev;
    h.alpha = -1.0; h.beta = 1.0; h.Cin = X; h.ldcin = ldx; h.C = X; h.ldc = ldx;
    // split-K as for the next-panel update (same m x b, K = 2 * nprev shape): the 128 x 64 tile grid alone is
    // about one wave (measured: zy 161 -> 147 ms per step at n = 32768); TRID_XUPD_SPLIT=0 turns it off (A/B)
    static const bool xsplit = !(getenv("TRID_XUPD_SPLIT") && getenv("TRID_XUPD_SPLIT")[0] == '0');
    if (xsplit) {
      h.splits = ws_skinny_splits(m, kk, 2 * nprev);
      if ((int64_t)h.splits * m * kk > part_elems) h.splits = 1;
      h.part = part; h.part_ld = m; h.part_stride = m * kk;
    }
    if ((e = gemm_ws(h, OP_N, st)) != cudaSuccess) return e;
  }
  // S = W^T X
  GemmArgs s;
  s.M = kk; s.N = kk; s.K[0] = m; s.A[0] = Wp; s.lda[0] = ldw; s.B[0] = X; s.ldb[0] = ldx;
  s.C = S; s.ldc = lds; s.alpha = 1.0; s.beta = 0.0;
  s.splits = pick_splits(kk, kk, m, TILE_64x64, part_elems);
  s.part = part; s.part_ld = kk; s.part_stride = (int64_t)kk * kk;
  (void)sem;   // in-kernel last-split reduction measured slower here (serial tail per tile); kept off
  static const bool s_ws = getenv("TRID_ZY_WS") && getenv("TRID_ZY_WS")[0] == '2';
  if (s_ws) {
    if ((e = gemm_ws_mm(OP_T, OP_N, kk, kk, m, 1.0, Wp, ldw, X, ldx, 0.0, S, lds, part, part_elems, st)) != cudaSuccess)
      return e;
  } else if ((e = gemm(s, OP_T, OP_N, TILE_64x64, st)) != cudaSuccess) {
    return e;
  }
  // Z_p = X - 1/2 Y_p S
  GemmArgs z;
  z.M = m; z.N = kk; z.K[0] = kk; z.A[0] = Yp; z.lda[0] = ldyz; z.B[0] = S; z.ldb[0] = lds;
  z.alpha = -0.5; z.beta = 1.0; z.Cin = X; z.ldcin = ldx; z.C = Zp; z.ldc = ldyz;
  return gemm_skinny_k(z, st);
}
}  // namespace trid

namespace {
// ---- the Z builder for one panel (a3): X = A W (SYMM); then zy_tail
cudaError_t zy_panel(int64_t m, int kk, const double* Atr, int64_t lda, const double* Wp, int64_t ldw,
                     const double* Yp, const double* Yprev, const double* Zprev, int64_t ldyz, int64_t nprev,
                     double* Zp, double* X, int64_t ldx, double* U, int64_t ldu, double* S, int64_t lds,
                     double* part, int64_t part_elems, unsigned* sem, cudaStream_t st) {
  cudaError_t e;
  // Default: the corrections X -= Y_< U1 + Z_< U2 ride in the SYMM launch as two extra K segments (U computed
  // first, negated); TRID_ZY_FOLD=0 keeps them as a separate split-K launch after the SYMM (zy_tail).
  static const bool fold = !(getenv("TRID_ZY_FOLD") && getenv("TRID_ZY_FOLD")[0] == '0') &&
                           !(getenv("TRID_ZY_WS") && getenv("TRID_ZY_WS")[0] == '0');
  const bool folded = fold && nprev > 0;
  if (folded) {
    double* U1 = U;
    double* U2 = U + nprev;
    {
      ProfScope ps(PROF_ZY, st);
      // [U1; U2] = -[Z_<^T W; Y_<^T W]   (TN, K = m, deterministic split-K): ONE launch over the stacked operands
      // (they share W; U2 = U1 + nprev in U's column); TRID_ZY_USTACK=0 runs the two products separately (A/B)
      static const bool ustack = !(getenv("TRID_ZY_USTACK") && getenv("TRID_ZY_USTACK")[0] == '0');
      if (ustack) {
        if ((e = gemm_ws_mm(OP_T, OP_N, 2 * nprev, kk, m, -1.0, Zprev, ldyz, Wp, ldw, 0.0, U1, ldu, part, part_elems,
                            st, Yprev, nprev)) != cudaSuccess)
          return e;
      } else {
        if ((e = gemm_ws_mm(OP_T, OP_N, nprev, kk, m, -1.0, Zprev, ldyz, Wp, ldw, 0.0, U1, ldu, part, part_elems,
                            st)) != cudaSuccess)
          return e;
        if ((e = gemm_ws_mm(OP_T, OP_N, nprev, kk, m, -1.0, Yprev, ldyz, Wp, ldw, 0.0, U2, ldu, part, part_elems,
                            st)) != cudaSuccess)
          return e;
      }
    }
    ProfScope ps(PROF_SYMM, st);
    e = symm_ws(m, kk, Atr, lda, Wp, ldw, X, ldx, part, part_elems, st, nprev, Yprev, U1, Zprev, U2, ldyz, ldu);
  } else {
    ProfScope ps(PROF_SYMM, st);
    e = symm_ws(m, kk, Atr, lda, Wp, ldw, X, ldx, part, part_elems, st);
  }
  if (e != cudaSuccess) return e;
  return zy_tail(m, kk, Wp, ldw, Yp, Yprev, Zprev, ldyz, nprev, Zp, X, ldx, U, ldu, S, lds, part, part_elems, sem, st,
                 folded);
}

int check_common(int64_t n, const void* A, int64_t lda, int b) {
  if (n < 0) return -1;
  if (n > 0 && A == nullptr) return -2;
  if (lda < (n > 1 ? n : 1)) return -3;
  if (b < 1) return -4;
  return 0;
}

}  // namespace


namespace {
char g_last_error[512] = "no error";
}
namespace trid {
void record_cuda_error(cudaError_t e, const char* what) {
  snprintf(g_last_error, sizeof g_last_error, "%s: %s (%d) in %s", cudaGetErrorName(e), cudaGetErrorString(e), (int)e,
           what);
}
void count_launches(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
void prof_mark(int cls, bool begin, cudaStream_t st) {
  ProfState& p = prof();
  if (!p.on) return;
  std::lock_guard<std::mutex> lk(p.mu);
  cudaEvent_t ev = prof_event(p);
  if (!ev) return;
  cudaEventRecord(ev, st);
  if (begin) {
    p.open[cls] = ev;
  } else if (p.open[cls]) {
    p.begins[cls].push_back(p.open[cls]);
    p.ends[cls].push_back(ev);
    p.open[cls] = nullptr;
  }
}
}  // namespace trid

extern "C" {

const char* trid_status_string(int status) {
  static char buf[64];
  switch (status) {
    case TRID_SUCCESS: return "success";
    case TRID_ERR_CUDA: return "CUDA error";
    case TRID_ERR_NCCL: return "NCCL error";
    case TRID_ERR_WORKSPACE: return "workspace too small";
    case TRID_ERR_UNSUPPORTED: return "unsupported configuration";
    default:
      if (status < 0) {
        snprintf(buf, sizeof buf, "invalid argument %d", -status);
        return buf;
      }
      return "unknown status";
  }
}

int trid_profile_begin(void) {
  ProfState& p = prof();
  std::lock_guard<std::mutex> lk(p.mu);
  p.on = true;
  p.used = 0;
  for (int c = 0; c < PROF_NCLASS; ++c) {
    p.open[c] = nullptr;
    p.begins[c].clear();
    p.ends[c].clear();
  }
  return TRID_SUCCESS;
}

int trid_profile_end(double* ms, int64_t* calls, int nclass) {
  ProfState& p = prof();
  std::lock_guard<std::mutex> lk(p.mu);
  p.on = false;
  for (int c = 0; c < nclass; ++c) {
    if (ms) ms[c] = 0.0;
    if (calls) calls[c] = 0;
  }
  for (int c = 0; c < PROF_NCLASS && c < nclass; ++c) {
    for (size_t i = 0; i < p.begins[c].size(); ++i) {
      float t = 0.f;
      if (cudaEventSynchronize(p.ends[c][i]) != cudaSuccess) return TRID_ERR_CUDA;
      if (cudaEventElapsedTime(&t, p.begins[c][i], p.ends[c][i]) != cudaSuccess) return TRID_ERR_CUDA;
      if (ms) ms[c] += t;
      if (calls) calls[c] += 1;
    }
  }
  return TRID_SUCCESS;
}

int64_t trid_kernel_launches(void) { return (int64_t)g_launches.load(); }

const char* trid_last_error_string(void) { return g_last_error; }

const char* trid_version(void) { return "trid-b200 0.1 sm_100a"; }

int trid_default_k(int64_t n, int b) { return b < 1 ? 0 : default_k(n, b); }

int64_t trid_bc_total_steps(int64_t n, int b) { return bc_total_steps(n, b); }

int trid_sbr_dbbr_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (nb < 1 || nb > b || b % nb) return -3;
  if (k != 0 && (k < b || k % b)) return -4;
  if (!dwork_bytes) return -5;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (k == 0) k = default_k(n, b);
  *dwork_bytes = n >= b + 2 ? carve_dbbr(nullptr, n, b, k).bytes : 256;
  return TRID_SUCCESS;
}

int trid_bulge_chase_bufsize(int64_t n, int b, size_t* dwork_bytes, int64_t* v2_len, int64_t* tau2_len) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (!dwork_bytes) return -3;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  const int beff = (int)(b < n - 1 ? b : (n - 1 > 1 ? n - 1 : 1));
  *dwork_bytes = bc_work_bytes(n > 0 ? n : 1, beff);
  const int64_t tot = bc_total_steps(n, b);
  if (v2_len) *v2_len = tot * b;
  if (tau2_len) *tau2_len = tot;
  return TRID_SUCCESS;
}

int trid_sytrd_2stage_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes, int64_t* v2_len,
                              int64_t* tau2_len) {
  size_t a = 0, c = 0;
  int r = trid_sbr_dbbr_bufsize(n, b, nb, k, &a);
  if (r) return r;
  r = trid_bulge_chase_bufsize(n, b, &c, v2_len, tau2_len);
  if (r) return r;
  if (!dwork_bytes) return -6;
  *dwork_bytes = a > c ? a : c;
  return TRID_SUCCESS;
}

int trid_sbr_dbbr(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* tau1, void* dwork,
                  size_t dwork_bytes, cudaStream_t stream) {
  int r = check_common(n, A, lda, b);
  if (r) return r;
  if (nb < 1 || nb > b || b % nb) return -5;
  if (k != 0 && (k < b || k % b)) return -6;
  if (n > 0 && !tau1) return -7;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (k == 0) k = default_k(n, b);
  if (n == 0) return TRID_SUCCESS;
  TRID_CUDA_TRY(cudaMemsetAsync(tau1, 0, sizeof(double) * (size_t)n, stream));
  if (n < b + 2) return TRID_SUCCESS;  // already banded (R4f): nothing to reduce
  if (!dwork) return -8;
  DbbrWork w = carve_dbbr(dwork, n, b, k);
  if (dwork_bytes < w.bytes) return TRID_ERR_WORKSPACE;
  TRID_CUDA_TRY(cudaMemsetAsync(w.sem, 0, sizeof(unsigned) * 1024, stream));
  const int64_t ld = n;  // Y, Z, W, X leading dimension
  for (int64_t i = 0; i + b + 1 < n; i += k) {                     // l.1
    int64_t ncols = 0, jlast = i;
    for (int64_t j = i; j < i + k && j + b + 1 < n; j += b) {     // l.3
      const int64_t o = j + b, m = n - o;
      const int kk = (int)(m < b ? m : b);
      double* Yp = w.Y + o + ncols * ld;
      double* Zp = w.Z + o + ncols * ld;
      // l.5: panel QR (V in place, T, explicit Y_p)
      {
        ProfScope ps(PROF_PANEL, stream);
        TRID_CUDA_TRY(panel_qr(m, b, A + o + j * lda, lda, tau1 + j, w.T, b, Yp, ld, w.red, w.bar, stream));
      }
      // W_p = Y_p T
      {
        GemmArgs g;
        g.M = m; g.N = kk; g.K[0] = kk; g.A[0] = Yp; g.lda[0] = ld; g.B[0] = w.T; g.ldb[0] = b;
        g.C = w.W; g.ldc = ld;
        ProfScope ps(PROF_WY, stream);
        TRID_CUDA_TRY(gemm_skinny_k(g, stream));
      }
      // Z builder against the implicitly updated trailing matrix (R4e)
      TRID_CUDA_TRY(zy_panel(m, kk, A + o + o * lda, lda, w.W, ld, Yp, w.Y + o, w.Z + o, ld, ncols, Zp, w.X, ld,
                             w.U, 2 * k, w.S, b, w.part, w.part_elems, w.sem, stream));
      ncols += kk;                                                  // l.6
      jlast = j;
      const int64_t jn = j + b;
      const bool last = !(jn < i + k && jn + b + 1 < n);
      if (!last) {                                                  // l.8-12 (R4d)
        GemmArgs g;
        g.M = m; g.N = b; g.nseg = 2;
        g.A[0] = w.Z + o; g.lda[0] = ld; g.B[0] = w.Y + o; g.ldb[0] = ld; g.K[0] = ncols;
        g.A[1] = w.Y + o; g.lda[1] = ld; g.B[1] = w.Z + o; g.ldb[1] = ld; g.K[1] = ncols;
        g.alpha = -1.0; g.beta = 1.0;
        g.C = A + o + o * lda; g.ldc = lda; g.Cin = g.C; g.ldcin = lda;
        g.lower = 1; g.diag_off = 0;
        g.splits = ws_skinny_splits(m, b, 2 * ncols);
        if ((int64_t)g.splits * m * b > w.part_elems) g.splits = 1;
        g.part = w.part; g.part_ld = m; g.part_stride = m * b;
        ProfScope ps(PROF_NEXT, stream);
        TRID_CUDA_TRY(gemm_ws(g, OP_T, stream));
      }
    }
    const int64_t e = jlast + b;                                    // l.15
    if (e < n) {
      GemmArgs g;
      g.M = n - e; g.N = n - e; g.nseg = 2;
      g.A[0] = w.Y + e; g.lda[0] = ld; g.B[0] = w.Z + e; g.ldb[0] = ld; g.K[0] = ncols;
      g.A[1] = w.Z + e; g.lda[1] = ld; g.B[1] = w.Y + e; g.ldb[1] = ld; g.K[1] = ncols;
      g.alpha = -1.0; g.beta = 1.0;
      g.C = A + e + e * lda; g.ldc = lda; g.Cin = g.C; g.ldcin = lda;
      g.lower = 1; g.tri = 1;
      ProfScope ps(PROF_SYR2K, stream);
      TRID_CUDA_TRY(gemm_ws(g, OP_T, stream));
    }
  }
  return TRID_SUCCESS;
}

int trid_bulge_chase(int64_t n, int b, const double* A, int64_t lda, double* d, double* e, double* V2, double* tau2,
                     void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  int r = check_common(n, A, lda, b);
  if (r) return r;
  if (n > 0 && !d) return -5;
  if (n > 1 && !e) return -6;
  if ((V2 == nullptr) != (tau2 == nullptr)) return -7;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (n == 0) return TRID_SUCCESS;
  size_t need = 0;
  trid_bulge_chase_bufsize(n, b, &need, nullptr, nullptr);
  if (!dwork) return -9;
  if (dwork_bytes < need) return TRID_ERR_WORKSPACE;
  ProfScope ps(PROF_BC, stream);
  TRID_CUDA_TRY(bulge_chase(n, b, A, lda, d, e, V2, tau2, dwork, stream));
  return TRID_SUCCESS;
}

int trid_sytrd_2stage(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* d, double* e, double* tau1,
                      double* V2, double* tau2, void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  int r = check_common(n, A, lda, b);
  if (r) return r;
  if (nb < 1 || nb > b || b % nb) return -5;
  if (k != 0 && (k < b || k % b)) return -6;
  size_t need = 0;
  r = trid_sytrd_2stage_bufsize(n, b, nb, k, &need, nullptr, nullptr);
  if (r) return r;
  if (n > 0 && dwork_bytes < need) return TRID_ERR_WORKSPACE;
  r = trid_sbr_dbbr(n, A, lda, b, nb, k, tau1, dwork, dwork_bytes, stream);
  if (r) return r;
  return trid_bulge_chase(n, b, A, lda, d, e, V2, tau2, dwork, dwork_bytes, stream);
}

int trid_stebz_bufsize(int64_t n, size_t* dwork_bytes) {
  if (n < 0) return -1;
  if (!dwork_bytes) return -2;
  *dwork_bytes = stebz_work_bytes(n > 0 ? n : 1);
  return TRID_SUCCESS;
}

int trid_stebz(int64_t n, const double* d, const double* e, double* w, void* dwork, size_t dwork_bytes,
               cudaStream_t stream) {
  if (n < 0) return -1;
  if (n > 0 && !d) return -2;
  if (n > 1 && !e) return -3;
  if (n > 0 && !w) return -4;
  if (n == 0) return TRID_SUCCESS;
  if (!dwork) return -5;
  if (dwork_bytes < stebz_work_bytes(n)) return TRID_ERR_WORKSPACE;
  TRID_CUDA_TRY(stebz(n, d, e, w, dwork, stream));
  return TRID_SUCCESS;
}

namespace {
struct EigWork {
  double *d, *e, *tau1;
  void* inner;
  size_t inner_bytes, bytes;
};
EigWork carve_eig(void* base, int64_t n, size_t inner) {
  EigWork w;
  Carver c(base);
  w.d = c.take<double>((size_t)(n > 0 ? n : 1));
  w.e = c.take<double>((size_t)(n > 1 ? n - 1 : 1));
  w.tau1 = c.take<double>((size_t)(n > 0 ? n : 1));
  w.inner = c.take<char>(inner);
  w.inner_bytes = inner;
  w.bytes = c.off;
  return w;
}
}  // namespace

int trid_syevals_2stage_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes) {
  if (!dwork_bytes) return -5;
  size_t a = 0;
  int r = trid_sytrd_2stage_bufsize(n, b, nb, k, &a, nullptr, nullptr);
  if (r) return r;
  const size_t s = stebz_work_bytes(n > 0 ? n : 1);
  *dwork_bytes = carve_eig(nullptr, n, a > s ? a : s).bytes;
  return TRID_SUCCESS;
}

int trid_syevals_2stage(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* w, void* dwork,
                        size_t dwork_bytes, cudaStream_t stream) {
  int r = check_common(n, A, lda, b);
  if (r) return r;
  if (nb < 1 || nb > b || b % nb) return -5;
  if (k != 0 && (k < b || k % b)) return -6;
  if (n > 0 && !w) return -7;
  size_t need = 0;
  r = trid_syevals_2stage_bufsize(n, b, nb, k, &need);
  if (r) return r;
  if (n == 0) return TRID_SUCCESS;
  if (!dwork) return -8;
  if (dwork_bytes < need) return TRID_ERR_WORKSPACE;
  size_t a = 0;
  trid_sytrd_2stage_bufsize(n, b, nb, k, &a, nullptr, nullptr);
  const size_t s = stebz_work_bytes(n);
  EigWork ew = carve_eig(dwork, n, a > s ? a : s);
  r = trid_sytrd_2stage(n, A, lda, b, nb, k, ew.d, ew.e, ew.tau1, nullptr, nullptr, ew.inner, ew.inner_bytes, stream);
  if (r) return r;
  {
    ProfScope ps(PROF_EIG, stream);
    TRID_CUDA_TRY(stebz(n, ew.d, ew.e, w, ew.inner, stream));
  }
  return TRID_SUCCESS;
}

int trid_sbr_backtransform_bufsize(int64_t n, int b, int k, int64_t ncols, size_t* dwork_bytes) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (k != 0 && (k < b || k % b)) return -3;
  if (ncols < 0) return -4;
  if (!dwork_bytes) return -5;
  if (k == 0) k = sbr_bt_default_k(b);
  *dwork_bytes = sbr_backtransform_work_bytes(n > 0 ? n : 1, b, k, ncols);
  return TRID_SUCCESS;
}

int trid_sbr_backtransform(int64_t n, int b, int k, const double* A, int64_t lda, const double* tau1, int trans,
                           int64_t ncols, double* C, int64_t ldc, void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (k != 0 && (k < b || k % b)) return -3;
  if (n > 0 && !A) return -4;
  if (lda < (n > 1 ? n : 1)) return -5;
  if (n > 0 && !tau1) return -6;
  if (trans != 0 && trans != 1) return -7;
  if (ncols < 0) return -8;
  if (n > 0 && ncols > 0 && !C) return -9;
  if (ldc < (n > 1 ? n : 1)) return -10;
  if (k == 0) k = sbr_bt_default_k(b);
  if (n == 0 || ncols == 0) return TRID_SUCCESS;
  if (!dwork) return -11;
  if (dwork_bytes < sbr_backtransform_work_bytes(n, b, k, ncols)) return TRID_ERR_WORKSPACE;
  ProfScope ps(PROF_SBR_BT, stream);
  TRID_CUDA_TRY(sbr_backtransform(n, b, k, A, lda, tau1, trans, ncols, C, ldc, dwork, stream));
  return TRID_SUCCESS;
}

int trid_bc_backtransform(int64_t n, int b, const double* V2, const double* tau2, int trans, int64_t ncols, double* C,
                          int64_t ldc, cudaStream_t stream) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  const bool has = n >= 3 && b >= 2;   // otherwise the chase stored no reflector (Q2 = I)
  if (has && !V2) return -3;
  if (has && !tau2) return -4;
  if (trans != 0 && trans != 1) return -5;
  if (ncols < 0) return -6;
  if (n > 0 && ncols > 0 && !C) return -7;
  if (ldc < (n > 1 ? n : 1)) return -8;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (!has || ncols == 0) return TRID_SUCCESS;
  ProfScope ps(PROF_BC_BT, stream);
  TRID_CUDA_TRY(bc_backtransform(n, b, V2, tau2, trans, ncols, C, ldc, stream));
  return TRID_SUCCESS;
}

int trid_panel_qr_bufsize(int64_t m, int w, size_t* dwork_bytes) {
  if (m < 0) return -1;
  if (w < 1) return -2;
  if (!dwork_bytes) return -3;
  if (w > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  *dwork_bytes = align256(panel_red_bytes(w)) + 1024;
  return TRID_SUCCESS;
}

int trid_panel_qr(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt, double* Y,
                  int64_t ldy, void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  if (m < 0) return -1;
  if (w < 1) return -2;
  if (m > 0 && !P) return -3;
  if (ldp < (m > 1 ? m : 1)) return -4;
  if (m > 0 && (!tau || !T || !Y)) return -5;
  if (ldt < w) return -7;
  if (ldy < (m > 1 ? m : 1)) return -9;
  if (w > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  size_t need = 0;
  trid_panel_qr_bufsize(m, w, &need);
  if (!dwork || dwork_bytes < need) return TRID_ERR_WORKSPACE;
  Carver c(dwork);
  double* red = (double*)c.take<char>(panel_red_bytes(w));
  unsigned* bar = c.take<unsigned>(256);
  TRID_CUDA_TRY(panel_qr(m, w, P, ldp, tau, T, ldt, Y, ldy, red, bar, stream));
  return TRID_SUCCESS;
}

int trid_syr2k_lower(int64_t m, int64_t kk, double* C, int64_t ldc, const double* Y, int64_t ldy, const double* Z,
                     int64_t ldz, cudaStream_t stream) {
  if (m < 0) return -1;
  if (kk < 0) return -2;
  if (m > 0 && !C) return -3;
  if (ldc < (m > 1 ? m : 1)) return -4;
  if (m > 0 && kk > 0 && !Y) return -5;
  if (ldy < (m > 1 ? m : 1)) return -6;
  if (m > 0 && kk > 0 && !Z) return -7;
  if (ldz < (m > 1 ? m : 1)) return -8;
  if (m == 0 || kk == 0) return TRID_SUCCESS;
  GemmArgs g;
  g.M = m; g.N = m; g.nseg = 2;
  g.A[0] = Y; g.lda[0] = ldy; g.B[0] = Z; g.ldb[0] = ldz; g.K[0] = kk;
  g.A[1] = Z; g.lda[1] = ldz; g.B[1] = Y; g.ldb[1] = ldy; g.K[1] = kk;
  g.alpha = -1.0; g.beta = 1.0; g.C = C; g.ldc = ldc; g.Cin = C; g.ldcin = ldc;
  g.lower = 1; g.tri = 1;
  TRID_CUDA_TRY(gemm_ws(g, OP_T, stream));
  return TRID_SUCCESS;
}

int trid_zy_bufsize(int64_t m, int w, size_t* dwork_bytes) {
  if (m < 0) return -1;
  if (w < 1) return -2;
  if (!dwork_bytes) return -3;
  int64_t pe = symm_ws_part_elems(m, w);
  const int64_t tn = (int64_t)32 * w * w;
  if (pe < tn) pe = tn;
  *dwork_bytes = align256(sizeof(double) * (size_t)m * w) + align256(sizeof(double) * (size_t)w * w) +
                 align256(sizeof(double) * (size_t)pe);
  return TRID_SUCCESS;
}

int trid_zy(int64_t m, int w, const double* A, int64_t lda, const double* W, int64_t ldw, const double* Y, int64_t ldy,
            double* Z, int64_t ldz, void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  if (m < 0) return -1;
  if (w < 1) return -2;
  if (m > 0 && !A) return -3;
  if (lda < (m > 1 ? m : 1)) return -4;
  if (m > 0 && !W) return -5;
  if (ldw < (m > 1 ? m : 1)) return -6;
  if (m > 0 && !Y) return -7;
  if (ldy < (m > 1 ? m : 1)) return -8;
  if (m > 0 && !Z) return -9;
  if (ldz < (m > 1 ? m : 1)) return -10;
  if (m == 0) return TRID_SUCCESS;
  size_t need = 0;
  trid_zy_bufsize(m, w, &need);
  if (!dwork || dwork_bytes < need) return TRID_ERR_WORKSPACE;
  Carver c(dwork);
  double* X = c.take<double>((size_t)m * w);
  double* S = c.take<double>((size_t)w * w);
  int64_t pe = symm_ws_part_elems(m, w);
  if (pe < (int64_t)32 * w * w) pe = (int64_t)32 * w * w;
  double* part = c.take<double>((size_t)pe);
  // Eq. (1) with no earlier panels: Y and Z of this call are separate buffers (ldy, ldz)
  cudaError_t e;
  {
    ProfScope ps(PROF_SYMM, stream);
    e = symm_ws(m, w, A, lda, W, ldw, X, m, part, pe, stream);
  }
  if (e != cudaSuccess) return TRID_ERR_CUDA;
  GemmArgs s;
  s.M = w; s.N = w; s.K[0] = m; s.A[0] = W; s.lda[0] = ldw; s.B[0] = X; s.ldb[0] = m;
  s.C = S; s.ldc = w; s.splits = pick_splits(w, w, m, TILE_64x64, pe);
  s.part = part; s.part_ld = w; s.part_stride = (int64_t)w * w;
  TRID_CUDA_TRY(gemm(s, OP_T, OP_N, TILE_64x64, stream));
  GemmArgs z;
  z.M = m; z.N = w; z.K[0] = w; z.A[0] = Y; z.lda[0] = ldy; z.B[0] = S; z.ldb[0] = w;
  z.alpha = -0.5; z.beta = 1.0; z.Cin = X; z.ldcin = m; z.C = Z; z.ldc = ldz;
  TRID_CUDA_TRY(gemm_ws(z, OP_N, stream));
  return TRID_SUCCESS;
}

}  // extern "C"
