// prof.cuh — optional stage timing (CUDA events on the caller's stream) and a kernel-launch counter.
// Disabled unless trid_profile_begin() was called; then every hot-path stage is bracketed by a pair
// of events recorded on the stream it is launched on (trid.h: trid_profile_*).
#pragma once
#include <cuda_runtime.h>

namespace trid {

enum ProfClass {
  PROF_PANEL = 0,   // a1/a2 panel QR (+T, Y)
  PROF_WY = 1,      // W = Y T
  PROF_SYMM = 2,    // a3 X = A W (SYMM, incl. split-K reduction)
  PROF_ZY = 3,      // a3 corrections, W^T X, Z = X - 1/2 Y S
  PROF_NEXT = 4,    // a4 next-panel update
  PROF_SYR2K = 5,   // a5 deferred syr2k
  PROF_BC = 6,      // a6+a7 band pack, bulge chase, d/e extraction
  PROF_EIG = 7,     // f3 Sturm bisection of T
  PROF_SBR_BT = 8,  // f1 SBR back-transformation (C <- Q1 C)
  PROF_BC_BT = 9,   // f2 BC back-transformation (C <- Q2 C)
  PROF_NCLASS = 10
};

void prof_mark(int cls, bool begin, cudaStream_t st);
void count_launches(int n);

struct ProfScope {
  int cls;
  cudaStream_t st;
  ProfScope(int c, cudaStream_t s) : cls(c), st(s) { prof_mark(cls, true, st); }
  ~ProfScope() { prof_mark(cls, false, st); }
};

}  // namespace trid
