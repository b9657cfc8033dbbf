// mg.cu — multi-GPU stage 1: DBBR (Alg. 1) with
// the trailing matrix 1D block-cyclic over column blocks of width b across the ranks of a communicator,
// one process (or, for tests, one host thread) per rank.
//
// Rank q of g owns global column blocks B with B % g == q, stored contiguously as its local columns
// (lda >= n: every rank stores full-height columns, only the lower triangle is referenced).  Per panel p
// at global column j (owner = (j/b) % g), with o = j+b, m = n-o:
//   owner : panel QR of its local panel columns -> packet [Y_p (m x kk) | T (b x b) | tau (kk)]
//   all   : broadcast(packet, owner)                           (the panel's V/T: "V/W broadcast")
//   all   : W_p = Y_p T; partial X_q = (lower entries this rank stores of A_blk) W_p
//             rows part : X(r)    += sum_{local x, cmap(x) <= r} A_loc(r, x) W(cmap(x))
//             cols part : X(c(x)) += sum_{r > c(x)}             A_loc(r, x) W(r)
//   all   : all-reduce(X, sum); Z builder tail (corrections, S, Z_p) redundantly on every rank
//   owner of the next panel's columns: next-panel update (Alg. 1 l.8-12)
// per outer block, every rank: syr2k on its own trailing columns (lower part), no communication.
// Y and Z are replicated (n x k each).  Collectives go through a small communicator: NCCL (dlopen'ed
// libnccl.so.2 — the one torch already loaded) or "local" virtual ranks in one process sharing a device
// (host-thread rendezvous + device copies; used to test the sharded arithmetic on a single GPU).
#include <dlfcn.h>
#include <nccl.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <condition_variable>
#include <memory>
#include <mutex>
#include <vector>

#include "../../include/trid.h"
#include "common.cuh"
#include "driver.cuh"
#include "gemm.cuh"
#include "panel.cuh"
#include "prof.cuh"

using namespace trid;

// ------------------------------------------------------------------------------------------------
// communicator
namespace {

struct NcclApi {
  bool ok = false;
  char err[256] = "";
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*reduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*getErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* path = getenv("TRID_NCCL_LIB");
    void* h = dlopen(path ? path : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      snprintf(api.err, sizeof api.err, "dlopen(%s): %s", path ? path : "libnccl.so.2", dlerror());
      return;
    }
#define TRID_SYM(field, name)                                                 \
  api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name));          \
  if (!api.field) {                                                           \
    snprintf(api.err, sizeof api.err, "dlsym(%s) failed", name);              \
    return;                                                                   \
  }
    TRID_SYM(getUniqueId, "ncclGetUniqueId");
    TRID_SYM(commInitRank, "ncclCommInitRank");
    TRID_SYM(commDestroy, "ncclCommDestroy");
    TRID_SYM(broadcast, "ncclBroadcast");
    TRID_SYM(allReduce, "ncclAllReduce");
    TRID_SYM(reduce, "ncclReduce");
    TRID_SYM(getErrorString, "ncclGetErrorString");
#undef TRID_SYM
    api.ok = true;
  });
  return api;
}

constexpr int kMaxLocal = 16;

// fixed-order sum of up to kMaxLocal device buffers into dst (dst may alias src[0])
struct SumPtrs {
  const double* p[kMaxLocal];
};
__global__ void sum_ptrs_kernel(double* dst, SumPtrs s, int g, int64_t count) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
    double v = s.p[0][i];
    for (int q = 1; q < g; ++q) v += s.p[q][i];
    dst[i] = v;
  }
}

// Virtual ranks in one process: every collective is a host rendezvous of the g calling threads plus
// stream-ordered device work, with the same semantics as the NCCL call it stands for.
struct LocalGroup {
  int g;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  std::vector<void*> ptr;
  std::vector<cudaEvent_t> ready, done;
  cudaEvent_t sum_ev = nullptr;
  explicit LocalGroup(int g_) : g(g_), ptr(g_), ready(g_), done(g_) {}
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const uint64_t my = gen;
    if (++arrived == g) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != my; });
    }
  }
};

}  // namespace

struct trid_comm {
  int kind = 0;   // 0 NCCL, 1 local virtual rank
  int nranks = 1, rank = 0;
  ncclComm_t nc = nullptr;
  std::shared_ptr<LocalGroup> grp;
};

namespace {

cudaError_t launch_sum(double* dst, const std::vector<void*>& src, int g, int64_t count, cudaStream_t st) {
  SumPtrs s{};
  for (int q = 0; q < g; ++q) s.p[q] = (const double*)src[q];
  int blocks = (int)((count + 255) / 256);
  if (blocks > 8 * num_sms()) blocks = 8 * num_sms();
  if (blocks < 1) blocks = 1;
  sum_ptrs_kernel<<<blocks, 256, 0, st>>>(dst, s, g, count);
  count_launches(1);
  return cudaGetLastError();
}

int nccl_status(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return TRID_SUCCESS;
  char buf[256];
  snprintf(buf, sizeof buf, "%s: %s", what, nccl().getErrorString ? nccl().getErrorString(r) : "nccl error");
  record_cuda_error(cudaErrorUnknown, buf);
  return TRID_ERR_NCCL;
}

// broadcast count doubles of buf from root (in place)
int comm_bcast(trid_comm* c, double* buf, int64_t count, int root, cudaStream_t st) {
  if (c->nranks == 1 || count <= 0) return TRID_SUCCESS;
  if (c->kind == 0) return nccl_status(nccl().broadcast(buf, buf, (size_t)count, ncclFloat64, root, c->nc, st), "ncclBroadcast");
  LocalGroup& G = *c->grp;
  const int q = c->rank;
  TRID_CUDA_TRY(cudaEventRecord(G.ready[q], st));
  G.ptr[q] = buf;
  G.barrier();
  if (q != root) {
    TRID_CUDA_TRY(cudaStreamWaitEvent(st, G.ready[root], 0));
    TRID_CUDA_TRY(cudaMemcpyAsync(buf, G.ptr[root], sizeof(double) * (size_t)count, cudaMemcpyDeviceToDevice, st));
    TRID_CUDA_TRY(cudaEventRecord(G.done[q], st));
  }
  G.barrier();
  if (q == root)
    for (int p = 0; p < G.g; ++p)
      if (p != root) TRID_CUDA_TRY(cudaStreamWaitEvent(st, G.done[p], 0));
  return TRID_SUCCESS;
}

// sum over ranks of count doubles; all == true: every rank gets the sum (all-reduce), else only root
int comm_sum(trid_comm* c, double* buf, int64_t count, bool all, int root, cudaStream_t st) {
  if (c->nranks == 1 || count <= 0) return TRID_SUCCESS;
  if (c->kind == 0) {
    if (all) return nccl_status(nccl().allReduce(buf, buf, (size_t)count, ncclFloat64, ncclSum, c->nc, st), "ncclAllReduce");
    return nccl_status(nccl().reduce(buf, buf, (size_t)count, ncclFloat64, ncclSum, root, c->nc, st), "ncclReduce");
  }
  LocalGroup& G = *c->grp;
  const int q = c->rank;
  TRID_CUDA_TRY(cudaEventRecord(G.ready[q], st));
  G.ptr[q] = buf;
  G.barrier();
  if (q == root) {
    for (int p = 0; p < G.g; ++p)
      if (p != root) TRID_CUDA_TRY(cudaStreamWaitEvent(st, G.ready[p], 0));
    std::vector<void*> src(G.g);
    src[0] = G.ptr[root];   // fixed order: root first, then the others by rank
    for (int p = 0, i = 1; p < G.g; ++p)
      if (p != root) src[i++] = G.ptr[p];
    TRID_CUDA_TRY(launch_sum(buf, src, G.g, count, st));
    TRID_CUDA_TRY(cudaEventRecord(G.sum_ev, st));
  }
  G.barrier();
  if (q != root) {
    TRID_CUDA_TRY(cudaStreamWaitEvent(st, G.sum_ev, 0));   // our buffer is read by the sum
    if (all) {
      TRID_CUDA_TRY(cudaMemcpyAsync(buf, G.ptr[root], sizeof(double) * (size_t)count, cudaMemcpyDeviceToDevice, st));
      TRID_CUDA_TRY(cudaEventRecord(G.done[q], st));
    }
  }
  G.barrier();
  if (q == root && all)
    for (int p = 0; p < G.g; ++p)
      if (p != root) TRID_CUDA_TRY(cudaStreamWaitEvent(st, G.done[p], 0));
  return TRID_SUCCESS;
}

// ------------------------------------------------------------------------------------------------
// block-cyclic column bookkeeping (host)
int64_t local_cols(int64_t n, int cb, int g, int q) {
  const int64_t nblk = (n + cb - 1) / cb;
  if (nblk <= q) return 0;
  const int64_t own = (nblk - q + g - 1) / g;
  int64_t cols = own * cb;
  if ((nblk - 1) % g == q) cols -= nblk * cb - n;   // the last (partial) block is ours
  return cols;
}
// number of local columns whose global index is < c0 (c0 a multiple of cb)
int64_t local_before(int64_t c0, int cb, int g, int q) {
  const int64_t B = c0 / cb;
  return (B > q ? (B - q + g - 1) / g : 0) * cb;
}
int64_t local_col(int64_t c, int cb, int g) { return (c / cb) / g * cb + c % cb; }

__device__ __forceinline__ int64_t mg_cmap(const MgMap& m, int64_t x) {
  const int64_t X = x + m.lofs, blk = X / m.cb;
  return (blk * m.g + m.q) * m.cb + (X - blk * m.cb) - m.gofs;
}
// dst(x, c) = src(cmap(x), c)
__global__ void gather_rows_kernel(double* dst, int64_t lddst, const double* src, int64_t ldsrc, int64_t rows,
                                   int64_t cols, MgMap mp) {
  const int64_t total = rows * cols;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = i % rows, c = i / rows;
    dst[x + c * lddst] = src[mg_cmap(mp, x) + c * ldsrc];
  }
}
// dst(cmap(x), c) += src(x, c)
__global__ void scatter_add_rows_kernel(double* dst, int64_t lddst, const double* src, int64_t ldsrc, int64_t rows,
                                        int64_t cols, MgMap mp) {
  const int64_t total = rows * cols;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = i % rows, c = i / rows;
    double* p = dst + mg_cmap(mp, x) + c * lddst;
    *p += src[x + c * ldsrc];
  }
}
// AB(o, c) = A(c+o, c) for this rank's columns c (LAPACK lower band storage), 0 <= o <= b
__global__ void band_scatter_kernel(double* AB, int64_t ldab, int64_t n, int b, const double* A, int64_t lda,
                                    int64_t nq, MgMap mp) {
  const int64_t total = nq * (b + 1);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = i / (b + 1), o = i % (b + 1);
    const int64_t c = mg_cmap(mp, x);
    if (c + o < n) AB[o + c * ldab] = A[(c + o) + x * lda];
  }
}

int grid_for(int64_t total) {
  int64_t blocks = (total + 255) / 256;
  if (blocks > 8 * num_sms()) blocks = 8 * num_sms();
  return blocks < 1 ? 1 : (int)blocks;
}

size_t align256(size_t x) { return (x + 255) / 256 * 256; }
// leading dimensions of the gathered operands are padded to 8 doubles so the DMMA engine's 16-byte loads apply
int64_t pad8(int64_t x) { return (x + 7) / 8 * 8; }
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

struct MgWork {
  double *Y, *Z, *W, *X, *Xl, *Wl, *Yl, *Zl, *T, *U, *S, *pk, *part, *red;
  unsigned *bar, *sem;
  int64_t part_elems;
  size_t bytes;
};

MgWork carve_mg(void* base, int64_t n, int b, int k, int g, int q) {
  const int64_t nq = local_cols(n, b, g, q);
  int64_t pe = (int64_t)32 * k * b;
  {
    const int64_t e = (int64_t)16 * (n - b) * b;   // skinny split-K bound (<= 16 splits, M <= n - b)
    if (e > pe) pe = e;
  }
  for (int64_t j = 0; j + b + 1 < n; j += b) {
    const int64_t o = j + b, m = n - o, kk = m < b ? m : b;
    const int64_t nqt = nq - local_before(o, b, g, q);
    if (nqt > 0) {
      const int64_t e = symm_mg_part_elems(m, kk, nqt);
      if (e > pe) pe = e;
    }
  }
  MgWork w;
  Carver c(base);
  w.Y = c.take<double>((size_t)n * k);
  w.Z = c.take<double>((size_t)n * k);
  w.W = c.take<double>((size_t)n * b);
  w.X = c.take<double>((size_t)pad8(n) * b);
  const size_t nqp = (size_t)pad8(nq > 0 ? nq : 1);
  w.Xl = c.take<double>(nqp * b);
  w.Wl = c.take<double>(nqp * b);
  w.Yl = c.take<double>(nqp * k);
  w.Zl = c.take<double>(nqp * k);
  w.T = c.take<double>((size_t)b * b);
  w.U = c.take<double>((size_t)2 * k * b);   // [Z_<^T W; Y_<^T W], ld 2k
  w.S = c.take<double>((size_t)b * b);
  w.pk = c.take<double>((size_t)n * b + (size_t)b * b + b);
  w.part_elems = pe;
  w.part = c.take<double>((size_t)pe);
  w.red = (double*)c.take<char>(panel_red_bytes(b));
  w.bar = c.take<unsigned>(256);   // panel grid-barrier counters (8 x 128 B)
  w.sem = c.take<unsigned>(1024);
  w.bytes = c.off;
  return w;
}

int default_k_mg(int b) {
  const int cap = b > 1024 ? b : 1024;
  return cap / b * b;
}

}  // namespace

extern "C" {

int trid_comm_unique_id(unsigned char id[128]) {
  if (!id) return -1;
  NcclApi& api = nccl();
  if (!api.ok) {
    record_cuda_error(cudaErrorUnknown, api.err);
    return TRID_ERR_NCCL;
  }
  ncclUniqueId u;
  const int r = nccl_status(api.getUniqueId(&u), "ncclGetUniqueId");
  if (r) return r;
  memcpy(id, u.internal, 128);
  return TRID_SUCCESS;
}

int trid_comm_init_nccl(const unsigned char id[128], int nranks, int rank, trid_comm_t* comm) {
  if (!id) return -1;
  if (nranks < 1) return -2;
  if (rank < 0 || rank >= nranks) return -3;
  if (!comm) return -4;
  NcclApi& api = nccl();
  if (!api.ok) {
    record_cuda_error(cudaErrorUnknown, api.err);
    return TRID_ERR_NCCL;
  }
  ncclUniqueId u;
  memcpy(u.internal, id, 128);
  ncclComm_t nc = nullptr;
  const int r = nccl_status(api.commInitRank(&nc, nranks, u, rank), "ncclCommInitRank");
  if (r) return r;
  trid_comm* c = new trid_comm;
  c->kind = 0;
  c->nranks = nranks;
  c->rank = rank;
  c->nc = nc;
  *comm = c;
  return TRID_SUCCESS;
}

int trid_comm_init_local(int nranks, trid_comm_t* comms) {
  if (nranks < 1 || nranks > kMaxLocal) return -1;
  if (!comms) return -2;
  auto grp = std::make_shared<LocalGroup>(nranks);
  TRID_CUDA_TRY(cudaEventCreateWithFlags(&grp->sum_ev, cudaEventDisableTiming));
  for (int q = 0; q < nranks; ++q) {
    TRID_CUDA_TRY(cudaEventCreateWithFlags(&grp->ready[q], cudaEventDisableTiming));
    TRID_CUDA_TRY(cudaEventCreateWithFlags(&grp->done[q], cudaEventDisableTiming));
  }
  for (int q = 0; q < nranks; ++q) {
    trid_comm* c = new trid_comm;
    c->kind = 1;
    c->nranks = nranks;
    c->rank = q;
    c->grp = grp;
    comms[q] = c;
  }
  return TRID_SUCCESS;
}

int trid_comm_destroy(trid_comm_t comm) {
  if (!comm) return -1;
  int r = TRID_SUCCESS;
  if (comm->kind == 0 && comm->nc) r = nccl_status(nccl().commDestroy(comm->nc), "ncclCommDestroy");
  if (comm->kind == 1 && comm->grp.use_count() == 1) {
    LocalGroup& G = *comm->grp;
    cudaEventDestroy(G.sum_ev);
    for (int q = 0; q < G.g; ++q) {
      cudaEventDestroy(G.ready[q]);
      cudaEventDestroy(G.done[q]);
    }
  }
  delete comm;
  return r;
}

int trid_comm_size(trid_comm_t comm) { return comm ? comm->nranks : -1; }
int trid_comm_rank(trid_comm_t comm) { return comm ? comm->rank : -1; }

int64_t trid_mg_local_cols(int64_t n, int colblock, int nranks, int rank) {
  if (n < 0 || colblock < 1 || nranks < 1 || rank < 0 || rank >= nranks) return -1;
  return local_cols(n, colblock, nranks, rank);
}

int trid_sbr_dbbr_mg_bufsize(int64_t n, int b, int nb, int k, int nranks, int rank, size_t* dwork_bytes) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (nb < 1 || nb > b || b % nb) return -3;
  if (k != 0 && (k < b || k % b)) return -4;
  if (nranks < 1) return -5;
  if (rank < 0 || rank >= nranks) return -6;
  if (!dwork_bytes) return -7;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (k == 0) k = default_k_mg(b);
  *dwork_bytes = n >= b + 2 ? carve_mg(nullptr, n, b, k, nranks, rank).bytes : 256;
  return TRID_SUCCESS;
}

int trid_sbr_dbbr_mg(trid_comm_t comm, int64_t n, double* A, int64_t lda, int colblock, int b, int nb, int k,
                     double* tau1, void* dwork, size_t dwork_bytes, cudaStream_t st) {
  if (!comm) return -1;
  if (n < 0) return -2;
  const int g = comm->nranks, q = comm->rank;
  const int64_t nq = local_cols(n, b > 0 ? b : 1, g, q);
  if (nq > 0 && !A) return -3;
  if (lda < (n > 1 ? n : 1)) return -4;
  if (colblock != b) return -5;
  if (b < 1) return -6;
  if (nb < 1 || nb > b || b % nb) return -7;
  if (k != 0 && (k < b || k % b)) return -8;
  if (n > 0 && !tau1) return -9;
  if (b > TRID_MAX_B) return TRID_ERR_UNSUPPORTED;
  if (k == 0) k = default_k_mg(b);
  if (n == 0) return TRID_SUCCESS;
  TRID_CUDA_TRY(cudaMemsetAsync(tau1, 0, sizeof(double) * (size_t)n, st));
  if (n < b + 2) return TRID_SUCCESS;
  if (!dwork) return -10;
  MgWork w = carve_mg(dwork, n, b, k, g, q);
  if (dwork_bytes < w.bytes) return TRID_ERR_WORKSPACE;
  TRID_CUDA_TRY(cudaMemsetAsync(w.sem, 0, sizeof(unsigned) * 1024, st));
  const int64_t ld = n;   // Y, Z, W leading dimension
  // row-sharded corrections (below); env TRID_MG_SHARD_CORR=0 (read per call, A/B and tests) repeats them per rank
  const bool shard_env = !(getenv("TRID_MG_SHARD_CORR") && getenv("TRID_MG_SHARD_CORR")[0] == '0');
  int r;
  for (int64_t i = 0; i + b + 1 < n; i += k) {                       // l.1
    int64_t ncols = 0, jlast = i;
    for (int64_t j = i; j < i + k && j + b + 1 < n; j += b) {       // l.3
      const int64_t o = j + b, m = n - o;
      const int kk = (int)(m < b ? m : b);
      const int owner = (int)((j / b) % g);
      double* pkY = w.pk;
      double* pkT = w.pk + (size_t)m * b;
      double* pkTau = pkT + (size_t)b * b;
      double* Yp = w.Y + o + ncols * ld;
      double* Zp = w.Z + o + ncols * ld;
      if (q == owner) {                                             // l.5 on the owner
        ProfScope ps(PROF_PANEL, st);
        TRID_CUDA_TRY(panel_qr(m, b, A + o + local_col(j, b, g) * lda, lda, pkTau, pkT, b, pkY, m, w.red, w.bar, st));
      }
      if ((r = comm_bcast(comm, w.pk, (int64_t)m * b + (int64_t)b * b + b, owner, st))) return r;
      TRID_CUDA_TRY(cudaMemcpy2DAsync(Yp, sizeof(double) * ld, pkY, sizeof(double) * m, sizeof(double) * m, kk,
                                      cudaMemcpyDeviceToDevice, st));
      TRID_CUDA_TRY(cudaMemcpyAsync(tau1 + j, pkTau, sizeof(double) * kk, cudaMemcpyDeviceToDevice, st));
      {                                                             // W_p = Y_p T
        GemmArgs gw;
        gw.M = m; gw.N = kk; gw.K[0] = kk; gw.A[0] = Yp; gw.lda[0] = ld; gw.B[0] = pkT; gw.ldb[0] = b;
        gw.C = w.W; gw.ldc = ld;
        ProfScope ps(PROF_WY, st);
        TRID_CUDA_TRY(gemm_ws(gw, OP_N, st));
      }
      // partial X over this rank's stored lower entries of the block-start trailing matrix, then all-reduce
      const int64_t lco = local_before(o, b, g, q), nqt = nq - lco, ldl = pad8(nqt), ldx = pad8(m);
      {
        ProfScope ps(PROF_SYMM, st);
        if (nqt > 0) {
          MgMap mp;
          mp.g = g; mp.q = q; mp.cb = b; mp.lofs = lco; mp.gofs = o;
          const double* Aq = A + o + lco * lda;
          gather_rows_kernel<<<grid_for(nqt * kk), 256, 0, st>>>(w.Wl, ldl, w.W, ld, nqt, kk, mp);
          count_launches(1);
          TRID_CUDA_TRY(cudaGetLastError());
          TRID_CUDA_TRY(symm_mg_rows(m, kk, nqt, Aq, lda, w.Wl, ldl, w.X, ldx, mp, w.part, w.part_elems, st));
          TRID_CUDA_TRY(symm_mg_cols(m, kk, nqt, Aq, lda, w.W, ld, w.Xl, ldl, mp, w.part, w.part_elems, st));
          scatter_add_rows_kernel<<<grid_for(nqt * kk), 256, 0, st>>>(w.X, ldx, w.Xl, ldl, nqt, kk, mp);
          count_launches(1);
          TRID_CUDA_TRY(cudaGetLastError());
        } else {
          TRID_CUDA_TRY(cudaMemsetAsync(w.X, 0, sizeof(double) * (size_t)ldx * kk, st));
        }
      }
      // Row-sharded corrections (R4e): every rank forms U = -[Z_<^T W; Y_<^T W] (Y, Z are replicated) and adds
      // Y_<(its row slice) U1 + Z_<(slice) U2 to its partial X, so the all-reduce returns the corrected X and the
      // correction GEMM (4 m b ncols flops per panel) is split over the g ranks instead of repeated on each one.
      // env TRID_MG_SHARD_CORR=0: every rank applies the whole correction after the all-reduce (zy_tail).
      const bool shard = shard_env && ncols > 0;
      if (shard) {
        ProfScope ps(PROF_ZY, st);
        double* U1 = w.U;
        double* U2 = w.U + ncols;
        // U = -[Z_<^T W; Y_<^T W] in one launch over the stacked operands (U2 = U1 + ncols)
        TRID_CUDA_TRY(gemm_ws_mm(OP_T, OP_N, 2 * ncols, kk, m, -1.0, w.Z + o, ld, w.W, ld, 0.0, U1, 2 * k, w.part,
                                 w.part_elems, st, w.Y + o, ncols));
        // contiguous row slices starting at even rows (16-byte aligned operands for the engine's fast producer)
        const int64_t rlo = q == 0 ? 0 : (m * q / g) & ~(int64_t)1;
        const int64_t rhi = q == g - 1 ? m : (m * (q + 1) / g) & ~(int64_t)1;
        if (rhi > rlo) {
          GemmArgs h;
          h.M = rhi - rlo; h.N = kk; h.nseg = 2;
          h.A[0] = w.Y + o + rlo; h.lda[0] = ld; h.B[0] = U1; h.ldb[0] = 2 * k; h.K[0] = ncols;
          h.A[1] = w.Z + o + rlo; h.lda[1] = ld; h.B[1] = U2; h.ldb[1] = 2 * k; h.K[1] = ncols;
          h.alpha = 1.0; h.beta = 1.0; h.Cin = w.X + rlo; h.ldcin = ldx; h.C = w.X + rlo; h.ldc = ldx;
          h.splits = ws_skinny_splits(rhi - rlo, kk, 2 * ncols);
          if ((int64_t)h.splits * (rhi - rlo) * kk > w.part_elems) h.splits = 1;
          h.part = w.part; h.part_ld = rhi - rlo; h.part_stride = (rhi - rlo) * kk;
          TRID_CUDA_TRY(gemm_ws(h, OP_N, st));
        }
      }
      {
        ProfScope ps(PROF_SYMM, st);
        if ((r = comm_sum(comm, w.X, ldx * kk, true, 0, st))) return r;   // padding rows ride along unread
      }
      TRID_CUDA_TRY(zy_tail(m, kk, w.W, ld, Yp, w.Y + o, w.Z + o, ld, ncols, Zp, w.X, ldx, w.U, 2 * k, w.S, b,
                            w.part, w.part_elems, w.sem, st, shard));
      ncols += kk;                                                  // l.6
      jlast = j;
      const int64_t jn = j + b;
      const bool last = !(jn < i + k && jn + b + 1 < n);
      if (!last && (int)((o / b) % g) == q) {                       // l.8-12 on the next panel's owner
        GemmArgs gn;
        gn.M = m; gn.N = b; gn.nseg = 2;
        gn.A[0] = w.Z + o; gn.lda[0] = ld; gn.B[0] = w.Y + o; gn.ldb[0] = ld; gn.K[0] = ncols;
        gn.A[1] = w.Y + o; gn.lda[1] = ld; gn.B[1] = w.Z + o; gn.ldb[1] = ld; gn.K[1] = ncols;
        gn.alpha = -1.0; gn.beta = 1.0;
        gn.C = A + o + local_col(o, b, g) * lda; gn.ldc = lda; gn.Cin = gn.C; gn.ldcin = lda;
        gn.lower = 1; gn.diag_off = 0;
        gn.splits = ws_skinny_splits(m, b, 2 * ncols);
        if ((int64_t)gn.splits * m * b > w.part_elems) gn.splits = 1;
        gn.part = w.part; gn.part_ld = m; gn.part_stride = m * b;
        ProfScope ps(PROF_NEXT, st);
        TRID_CUDA_TRY(gemm_ws(gn, OP_T, st));
      }
    }
    const int64_t e = jlast + b;                                    // l.15 on every rank's own columns
    const int64_t lce = local_before(e, b, g, q), nqe = nq - lce, lde = pad8(nqe);
    if (e < n && nqe > 0) {
      ProfScope ps(PROF_SYR2K, st);
      MgMap mp;
      mp.g = g; mp.q = q; mp.cb = b; mp.lofs = lce; mp.gofs = e;
      gather_rows_kernel<<<grid_for(nqe * ncols), 256, 0, st>>>(w.Yl, lde, w.Y + e, ld, nqe, ncols, mp);
      gather_rows_kernel<<<grid_for(nqe * ncols), 256, 0, st>>>(w.Zl, lde, w.Z + e, ld, nqe, ncols, mp);
      count_launches(2);
      TRID_CUDA_TRY(cudaGetLastError());
      GemmArgs gs;
      gs.M = n - e; gs.N = nqe; gs.nseg = 2;
      gs.A[0] = w.Y + e; gs.lda[0] = ld; gs.B[0] = w.Zl; gs.ldb[0] = lde; gs.K[0] = ncols;
      gs.A[1] = w.Z + e; gs.lda[1] = ld; gs.B[1] = w.Yl; gs.ldb[1] = lde; gs.K[1] = ncols;
      gs.alpha = -1.0; gs.beta = 1.0;
      gs.C = A + e + lce * lda; gs.ldc = lda; gs.Cin = gs.C; gs.ldcin = lda;
      gs.lower = 1;
      gs.mg_g = g; gs.mg_q = q; gs.mg_cb = b; gs.mg_lofs = lce; gs.mg_gofs = e;
      TRID_CUDA_TRY(gemm_ws(gs, OP_T, st));
    }
  }
  return TRID_SUCCESS;
}

int trid_band_gather(trid_comm_t comm, int64_t n, int b, const double* A, int64_t lda, int colblock, int root,
                     double* AB, int64_t ldab, cudaStream_t st) {
  if (!comm) return -1;
  if (n < 0) return -2;
  if (b < 1) return -3;
  const int g = comm->nranks, q = comm->rank;
  const int64_t nq = local_cols(n, colblock > 0 ? colblock : 1, g, q);
  if (nq > 0 && !A) return -4;
  if (lda < (n > 1 ? n : 1)) return -5;
  if (colblock < 1) return -6;
  if (root < 0 || root >= g) return -7;
  if (n > 0 && !AB) return -8;
  if (ldab < b + 1) return -9;
  if (n == 0) return TRID_SUCCESS;
  TRID_CUDA_TRY(cudaMemsetAsync(AB, 0, sizeof(double) * (size_t)ldab * n, st));
  if (nq > 0) {
    MgMap mp;
    mp.g = g; mp.q = q; mp.cb = colblock; mp.lofs = 0; mp.gofs = 0;
    band_scatter_kernel<<<grid_for(nq * (b + 1)), 256, 0, st>>>(AB, ldab, n, b, A, lda, nq, mp);
    count_launches(1);
    TRID_CUDA_TRY(cudaGetLastError());
  }
  return comm_sum(comm, AB, ldab * n, false, root, st);
}

int trid_bulge_chase_band(int64_t n, int b, const double* AB, int64_t ldab, double* d, double* e, double* V2,
                          double* tau2, void* dwork, size_t dwork_bytes, cudaStream_t stream) {
  if (n < 0) return -1;
  if (b < 1) return -2;
  if (n > 0 && !AB) return -3;
  if (ldab < b + 1) return -4;
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
  TRID_CUDA_TRY(bulge_chase_cs(n, b, AB, ldab, d, e, V2, tau2, dwork, stream));
  return TRID_SUCCESS;
}

}  // extern "C"
