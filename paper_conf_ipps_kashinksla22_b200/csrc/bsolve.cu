// bsolve.cu -- host side of the C ABI declared in include/bsolve.h.
//
// bsolve_create analyses the shared pattern once (validation, diagonal slot
// per row, ELL column indices, bandwidth) and chooses the kernel variant
// (format x placement x rows-per-thread x CTA size) and its dynamic shared
// memory -- the B200 analogue of the paper's automatic shared-memory
// configuration and block-size tuning (Sec. IV-D;
// PAPER.md:836-850, Sec. IV-E).  bsolve_run validates arguments and enqueues
// ONE kernel launch on the caller's stream.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdint>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/bsolve.h"
#include "banded.cuh"
#include "kernels.cuh"
#include "variants.h"

using namespace bsolve;

// ------------------------------------------------------------- errors --
static thread_local std::string g_err;

static int fail(int code, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define CUDA_TRY(call)                                                                    \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess)                                                                \
      return fail(BSOLVE_ERR_CUDA, "%s failed: %s", #call, cudaGetErrorString(e_));       \
  } while (0)

// ------------------------------------------------------- kernel table --
// The instantiations live in k_generic.cu / k_special.cu / k_line.cu
// (compiled in parallel); variants.h declares the tables.
static const PVariant *find_pvariant(int fmt, int r) {
  int cnt = 0;
  const PVariant *t = variants_persist(&cnt);
  for (int i = 0; i < cnt; ++i)
    if (t[i].fmt == fmt && t[i].r == r) return &t[i];
  return nullptr;
}

static const CVariant *find_cvariant(int c, int kreg, int rounds) {
  int cnt = 0;
  const CVariant *t = variants_cluster(&cnt);
  for (int i = 0; i < cnt; ++i)
    if (t[i].c == c && t[i].kreg == kreg && t[i].rounds == rounds) return &t[i];
  return nullptr;
}

static const Variant *find_variant(int fmt, int place, int wb, bool exact, int r, int nt,
                                   int kreg = 0) {
  int cnt = 0;
  const Variant *t = variants_generic(&cnt);
  for (int i = 0; i < cnt; ++i) {
    const Variant &v = t[i];
    if (v.fmt == fmt && v.place == place && v.wb == wb && v.exact == exact && v.r == r &&
        v.nt == nt && v.kreg == kreg)
      return &v;
  }
  return nullptr;
}

// ------------------------------------------------------------- handle --
struct bsolve_plan {
  int n = 0, nnz = 0, batch = 0, W = 0, wb = 0;
  int solver = 0, precond = 0, restart = 0;
  int fmt = 0, place = 0, stop = 0, trc = 1, device = 0;
  int nt = 0, r = 0, smem_bytes = 0, smem_vals = 0, n_pad = 0, ctas_per_sm = 0, num_sms = 0;
  int occ_api = 0;         // cudaOccupancyMaxActiveBlocksPerMultiprocessor (TMEM plans)
  int regs = 0;            // registers per thread of the solve kernel
  int kl = 0, ku = 0;
  int kfmt = 0;            // kernel storage mode: FMT_CSR / FMT_ELL / FMT_DIA
  int guard = 0;           // DIA: zero doubles around the gather body
  int doff[kMaxW] = {};    // DIA: byte offset of slot k
  long long sys_stride = 0;
  const Variant *var = nullptr;      // per-system-CTA kernel (also the REGS fallback)
  const PVariant *pvar = nullptr;    // persistent kernel when place == PLACE_REGS
  const CVariant *cvar = nullptr;    // cluster kernel when place == PLACE_CLUSTER
  solve_fn var_tmem = nullptr;       // TMEM kernel when place == PLACE_TMEM
  int line_nx = 0;                   // > 0: line-tiled TMEM kernel for an NX-wide 9-point grid
  int line_a = 0;                    // generic-width line kernel: line_nx / 8 (else 0)
  int line_generic = 0;              // 1: the generic-width line kernel
  int line_ctas = 0;                 // its resident CTAs per SM (launch bounds)
  int st_ok = 0;                     // pattern is a uniform-offset stencil (st_doff valid)
  int st_doff[kMaxW] = {};           // byte offset d_k * 8 of ELL slot k (stencils)
  int32_t *d_vidx = nullptr;         // CSR values on the line plan: [9][n] value index of
                                     // canonical slot c (8 = diagonal) of row r, -1 none
  int c2s[8] = {-1, -1, -1, -1, -1, -1, -1, -1};  // its canonical offset -> ELL slot map
  int cluster = 0;                   // CTAs per system (cluster plan)
  int smem_bytes_fallback = 0, grid_persist = 0;
  int max_clusters = 0;  // PLACE_CLUSTER: cudaOccupancyMaxActiveClusters
  unsigned long long *d_ctr = nullptr;  // persistent work counter + finished-CTA count
  std::vector<int32_t> h_ell_col;  // [W][n]
  std::vector<int32_t> h_csr2ell;  // [W][n] -> CSR entry held by the slot, -1 = padding
  int32_t *d_ell_col = nullptr, *d_row_ptr = nullptr, *d_diag = nullptr, *d_src = nullptr;
  // bsolve_run_host pipeline (lazily allocated)
  static constexpr int kSlots = 3;
  cudaStream_t hs[kSlots] = {nullptr, nullptr, nullptr};
  int h_chunk = 0;
  double *h_val[kSlots] = {}, *h_b[kSlots] = {}, *h_x0[kSlots] = {}, *h_x[kSlots] = {},
         *h_res[kSlots] = {};
  int32_t *h_it[kSlots] = {};
  int8_t *h_st[kSlots] = {};
  double *h_bws[kSlots] = {};       // banded workspace per pipeline slot
  size_t h_bws_bytes[kSlots] = {};
  double *h_fbws[kSlots] = {};      // direct fallback per pipeline slot: workspace,
  int32_t *h_fbl[kSlots] = {};      //   compacted system list (chunk entries),
  int32_t *h_fbn[kSlots] = {};      //   list length
  // banded direct solver (bsolve_banded_solve, lazily set up)
  int32_t *d_bnd = nullptr;   // [W][n] packed (value index << 8) | (col mod window width)
  int32_t *d_bcol = nullptr;  // [W][n] column of ELL slot k of row r (fallback residual)
  int bnd_w = 0;              // window width the table's ring positions use
  const BVariant *bvar = nullptr;  // banded instance covering the pattern (setup_banded)
  int smem_optin = 0;         // device limit on dynamic SMEM per CTA
  int direct_fallback = 0;    // bsolve_options.direct_fallback
  int banded_launches = 0;    // kernel launches of the last banded call
  double *d_bws = nullptr;    // split banded solve: per-system U + y workspace (one chunk)
  size_t bws_bytes = 0;
  // direct fallback (allocated by bsolve_create, so bsolve_run stays asynchronous):
  // fused-kernel workspace for fb_grid CTAs, the compacted list of non-converged
  // systems and its length
  int fb_grid = 0;
  double *d_fbws = nullptr;
  int32_t *d_fbl = nullptr, *d_fbn = nullptr;
};

static int setup_banded(bsolve_handle h);
static size_t banded_ws_sys(bsolve_handle h);
static int alloc_fallback(bsolve_handle h, int grid, long long list_len, double **ws,
                          int32_t **list, int32_t **len);

extern "C" void bsolve_default_options(bsolve_options *o) {
  if (!o) return;
  o->format = BSOLVE_FMT_AUTO;
  o->placement = BSOLVE_PLACE_AUTO;
  o->stop = BSOLVE_STOP_REL_B;
  o->true_residual_check = 1;
  o->device = -1;
  o->block_threads = 0;
  o->reg_slots = 0;
  o->solver = BSOLVE_SOLVER_BICGSTAB;
  o->precond = BSOLVE_PREC_JACOBI;
  o->restart = BSOLVE_MAX_RESTART;
  o->direct_fallback = 0;
}

static void free_plan(bsolve_plan *h) {
  if (!h) return;
  int cur = -1;
  cudaGetDevice(&cur);
  cudaSetDevice(h->device);
  cudaFree(h->d_ell_col);
  cudaFree(h->d_row_ptr);
  cudaFree(h->d_diag);
  cudaFree(h->d_src);
  cudaFree(h->d_ctr);
  cudaFree(h->d_bnd);
  cudaFree(h->d_bcol);
  cudaFree(h->d_vidx);
  cudaFree(h->d_bws);
  cudaFree(h->d_fbws);
  cudaFree(h->d_fbl);
  cudaFree(h->d_fbn);
  for (int s = 0; s < bsolve_plan::kSlots; ++s) {
    if (h->hs[s]) cudaStreamDestroy(h->hs[s]);
    cudaFree(h->h_val[s]);
    cudaFree(h->h_b[s]);
    cudaFree(h->h_x0[s]);
    cudaFree(h->h_x[s]);
    cudaFree(h->h_res[s]);
    cudaFree(h->h_it[s]);
    cudaFree(h->h_st[s]);
    cudaFree(h->h_bws[s]);
    cudaFree(h->h_fbws[s]);
    cudaFree(h->h_fbl[s]);
    cudaFree(h->h_fbn[s]);
  }
  if (cur >= 0) cudaSetDevice(cur);
  delete h;
}

// Validate the shared CSR pattern; fills diag slot per row. Pure host code.
static int validate_pattern(int n, const int32_t *rp, const int32_t *ci, std::vector<int32_t> &diag,
                            int &W) {
  if (rp[0] != 0) return fail(BSOLVE_ERR_PATTERN, "row_ptr[0] = %d, expected 0", rp[0]);
  diag.assign(n, -1);
  W = 0;
  for (int i = 0; i < n; ++i) {
    if (rp[i + 1] < rp[i])
      return fail(BSOLVE_ERR_PATTERN, "row_ptr decreases at row %d (%d -> %d)", i, rp[i], rp[i + 1]);
    W = std::max(W, rp[i + 1] - rp[i]);
    for (int e = rp[i]; e < rp[i + 1]; ++e) {
      const int c = ci[e];
      if (c < 0 || c >= n)
        return fail(BSOLVE_ERR_PATTERN, "col_idx[%d] = %d out of range [0, %d)", e, c, n);
      if (e > rp[i] && c <= ci[e - 1])
        return fail(BSOLVE_ERR_PATTERN, "row %d: columns not strictly increasing at entry %d", i, e);
      if (c == i) diag[i] = e - rp[i];
    }
    if (diag[i] < 0) return fail(BSOLVE_ERR_PATTERN, "row %d has no diagonal entry", i);
  }
  return BSOLVE_OK;
}

// ELL slot assignment (create time).  The paper's BatchEll stores each row's
// entries padded to a uniform width, column-major (PAPER.md:491-499,
// 522-524); it leaves the slot order free.  We choose it for conflict-free
// shared-memory gathers on B200: slot k is tied to the k-th most frequent
// column offset d_k = col - row of the pattern (for the 9-point stencil the
// 9 stencil offsets), so the 32 lanes of a warp (32 consecutive rows) read
// gather addresses row + d_k that are consecutive -> 2 wavefronts per
// LDS.64 instead of 4 at grid-boundary rows.  Entries whose offset is not a
// template offset take the remaining free slots; padding slots get a column
// congruent to row + d_k modulo 16 doubles (same bank pair) and value 0.
static void build_ell_map(int n, const int32_t *rp, const int32_t *ci, int W,
                          std::vector<int32_t> &ell_col, std::vector<int32_t> &src,
                          std::vector<int32_t> &ell_diag) {
  std::vector<std::pair<int, int>> hist;  // (offset, count)
  {
    std::vector<int> offs;
    offs.reserve(rp[n]);
    for (int i = 0; i < n; ++i)
      for (int e = rp[i]; e < rp[i + 1]; ++e) offs.push_back(ci[e] - i);
    std::sort(offs.begin(), offs.end());
    for (size_t a = 0; a < offs.size();) {
      size_t b = a;
      while (b < offs.size() && offs[b] == offs[a]) ++b;
      hist.push_back({offs[a], (int)(b - a)});
      a = b;
    }
  }
  std::stable_sort(hist.begin(), hist.end(), [](const std::pair<int, int> &x,
                                                const std::pair<int, int> &y) {
    if (x.second != y.second) return x.second > y.second;
    if (std::abs(x.first) != std::abs(y.first)) return std::abs(x.first) < std::abs(y.first);
    return x.first < y.first;
  });
  std::vector<int> tmpl;
  for (int k = 0; k < W && k < (int)hist.size(); ++k) tmpl.push_back(hist[k].first);
  std::sort(tmpl.begin(), tmpl.end());
  // the diagonal (offset 0, present in every row, hence in the template) goes
  // to slot 0: the kernels keep its value and its gather operand in registers
  tmpl.erase(std::find(tmpl.begin(), tmpl.end(), 0));
  tmpl.insert(tmpl.begin(), 0);
  while ((int)tmpl.size() < W) tmpl.push_back(0);
  ell_col.assign((size_t)W * n, 0);
  src.assign((size_t)W * n, -1);
  ell_diag.assign(n, 0);
  std::vector<int> slot_of(W);
  for (int i = 0; i < n; ++i) {
    std::vector<char> used(W, 0);
    std::vector<int> rest;
    for (int e = rp[i]; e < rp[i + 1]; ++e) {
      const int o = ci[e] - i;
      bool placed = false;
      for (int k = 0; k < W; ++k)  // tmpl is not sorted (offset 0 first)
        if (tmpl[k] == o && !used[k]) {
          used[k] = 1;
          src[(size_t)k * n + i] = e;
          ell_col[(size_t)k * n + i] = ci[e];
          placed = true;
          break;
        }
      if (!placed) rest.push_back(e);
    }
    size_t r = 0;
    for (int k = 0; k < W; ++k) {
      if (used[k]) continue;
      if (r < rest.size()) {
        const int e = rest[r++];
        used[k] = 1;
        src[(size_t)k * n + i] = e;
        ell_col[(size_t)k * n + i] = ci[e];
      } else {
        long long t = (long long)i + tmpl[k];
        long long c = t;
        if (t < 0) c = ((t % 16) + 16) % 16;
        else if (t >= n) c = t - 16 * ((t - (n - 1) + 15) / 16);
        if (c < 0 || c >= n) c = i;
        ell_col[(size_t)k * n + i] = (int32_t)c;
      }
    }
    for (int k = 0; k < W; ++k)
      if (src[(size_t)k * n + i] >= 0 && ell_col[(size_t)k * n + i] == i) ell_diag[i] = k;
  }
}

extern "C" int bsolve_ell_layout(int n, const int32_t *row_ptr, const int32_t *col_idx,
                                 int32_t *width, int32_t *cols, int32_t *src) {
  g_err.clear();
  if (n <= 0) return fail(BSOLVE_ERR_INVALID, "n = %d must be >= 1", n);
  if (!row_ptr || !col_idx || !width) return fail(BSOLVE_ERR_INVALID, "NULL argument");
  std::vector<int32_t> diag;
  int W = 0;
  int rc = validate_pattern(n, row_ptr, col_idx, diag, W);
  if (rc) return rc;
  *width = W;
  if (cols || src) {
    std::vector<int32_t> c, s, d;
    build_ell_map(n, row_ptr, col_idx, W, c, s, d);
    if (cols) std::memcpy(cols, c.data(), sizeof(int32_t) * c.size());
    if (src) std::memcpy(src, s.data(), sizeof(int32_t) * s.size());
  }
  return BSOLVE_OK;
}

extern "C" int bsolve_create(bsolve_handle *out, int n, int batch, const int32_t *row_ptr,
                             const int32_t *col_idx, const bsolve_options *opt_in) {
  g_err.clear();
  if (!out) return fail(BSOLVE_ERR_INVALID, "out is NULL");
  *out = nullptr;
  if (n <= 0) return fail(BSOLVE_ERR_INVALID, "n = %d must be >= 1", n);
  if (batch < 0) return fail(BSOLVE_ERR_INVALID, "batch = %d must be >= 0", batch);
  if (!row_ptr || !col_idx) return fail(BSOLVE_ERR_INVALID, "row_ptr/col_idx is NULL");
  bsolve_options opt;
  bsolve_default_options(&opt);
  if (opt_in) opt = *opt_in;
  if (opt.format < BSOLVE_FMT_AUTO || opt.format > BSOLVE_FMT_ELL)
    return fail(BSOLVE_ERR_INVALID, "bad format %d", opt.format);
  if (opt.placement < BSOLVE_PLACE_AUTO || opt.placement > BSOLVE_PLACE_TMEM)
    return fail(BSOLVE_ERR_INVALID, "bad placement %d", opt.placement);
  if (opt.stop != BSOLVE_STOP_REL_B && opt.stop != BSOLVE_STOP_ABS)
    return fail(BSOLVE_ERR_INVALID, "bad stop mode %d", opt.stop);
  if (opt.block_threads != 0 && opt.block_threads != 128 && opt.block_threads != 256 &&
      opt.block_threads != 512)
    return fail(BSOLVE_ERR_INVALID, "block_threads must be 0, 128, 256 or 512 (got %d)",
                opt.block_threads);
  if (opt.reg_slots < 0 || opt.reg_slots > 8 || (opt.reg_slots & 1))
    return fail(BSOLVE_ERR_INVALID, "reg_slots must be 0, 2, 4, 6 or 8 (got %d)", opt.reg_slots);
  if (opt.solver != BSOLVE_SOLVER_BICGSTAB && opt.solver != BSOLVE_SOLVER_GMRES)
    return fail(BSOLVE_ERR_INVALID, "bad solver %d", opt.solver);
  if (opt.precond != BSOLVE_PREC_JACOBI && opt.precond != BSOLVE_PREC_NONE &&
      opt.precond != BSOLVE_PREC_BLOCK_JACOBI)
    return fail(BSOLVE_ERR_INVALID, "bad preconditioner %d", opt.precond);
  if (opt.precond == BSOLVE_PREC_BLOCK_JACOBI && opt.solver != BSOLVE_SOLVER_BICGSTAB)
    return fail(BSOLVE_ERR_UNSUPPORTED, "block-Jacobi is implemented for BiCGSTAB only");
  if (opt.solver == BSOLVE_SOLVER_GMRES && (opt.restart < 1 || opt.restart > BSOLVE_MAX_RESTART))
    return fail(BSOLVE_ERR_INVALID, "GMRES restart must be 1..%d (got %d)", BSOLVE_MAX_RESTART,
                opt.restart);
  static_assert(BSOLVE_MAX_RESTART == kMaxRestart, "header and kernel restart bound");

  std::vector<int32_t> diag;
  int W = 0;
  int rc = validate_pattern(n, row_ptr, col_idx, diag, W);
  if (rc) return rc;
  const int nnz = row_ptr[n];
  if (W > 16)
    return fail(BSOLVE_ERR_UNSUPPORTED, "rows with %d > 16 entries are not supported", W);
  if ((long long)n * 8 >= 65536)
    return fail(BSOLVE_ERR_UNSUPPORTED, "n = %d too large (packed 16-bit gather offsets need n < 8192)", n);

  bsolve_plan *h = new (std::nothrow) bsolve_plan();
  if (!h) return fail(BSOLVE_ERR_NOMEM, "host allocation failed");
  h->n = n;
  h->nnz = nnz;
  h->batch = batch;
  h->W = W;
  h->wb = W == 9 ? 9 : 16;
  h->fmt = opt.format == BSOLVE_FMT_CSR ? FMT_CSR : FMT_ELL;
  h->stop = opt.stop;
  h->trc = opt.true_residual_check ? 1 : 0;
  h->solver = opt.solver;
  h->precond = opt.precond;
  h->restart = opt.solver == BSOLVE_SOLVER_GMRES ? opt.restart : 0;
  h->direct_fallback = opt.direct_fallback ? 1 : 0;
  h->sys_stride = h->fmt == FMT_ELL ? (long long)W * n : nnz;

  // bandwidth (for bsolve_info; the banded structure is not used by the solve)
  for (int i = 0; i < n; ++i)
    for (int e = row_ptr[i]; e < row_ptr[i + 1]; ++e) {
      h->kl = std::max(h->kl, i - col_idx[e]);
      h->ku = std::max(h->ku, col_idx[e] - i);
    }
  if (h->direct_fallback) {  // the banded kernels must cover the pattern (fail early)
    int cnt = 0;
    const BVariant *tab = variants_banded(&cnt);
    bool ok = false;
    for (int i = 0; i < cnt; ++i)
      ok = ok || (tab[i].kb >= std::max(h->kl, h->ku) && tab[i].max_entries > W);
    if (!ok) {
      const int kl = h->kl, ku = h->ku;
      delete h;
      return fail(BSOLVE_ERR_UNSUPPORTED,
                  "direct_fallback: bandwidth kl = %d, ku = %d exceeds the banded solver", kl, ku);
    }
  }
  // ELL slot map (conflict-free gathers, see build_ell_map)
  std::vector<int32_t> ell_diag;
  build_ell_map(n, row_ptr, col_idx, W, h->h_ell_col, h->h_csr2ell, ell_diag);
  if (h->fmt == FMT_ELL) diag = ell_diag;  // kernel needs the diagonal's slot in its format
  h->kfmt = h->fmt;
  {
    // DIA (uniform-offset) addressing if every real entry of slot k sits at
    // column row + d_k for one d_k per slot: true for stencil patterns.  A
    // property of the pattern (st_ok, st_doff: the line-tiled plans take it
    // for both value layouts); ELL values also switch the generic kernels to
    // DIA addressing.
    std::vector<long long> dk(W, LLONG_MIN);
    bool uniform = true;
    for (int k = 0; k < W && uniform; ++k)
      for (int i = 0; i < n; ++i) {
        if (h->h_csr2ell[(size_t)k * n + i] < 0) continue;
        const long long o = (long long)h->h_ell_col[(size_t)k * n + i] - i;
        if (dk[k] == LLONG_MIN) dk[k] = o;
        else if (dk[k] != o) { uniform = false; break; }
      }
    if (uniform && dk[0] == 0) {
      long long g = 0;
      for (int k = 0; k < W; ++k) {
        if (dk[k] == LLONG_MIN) dk[k] = 0;
        g = std::max<long long>(g, dk[k] < 0 ? -dk[k] : dk[k]);
        h->doff[k] = (int)(dk[k] * 8);
      }
      h->st_ok = 1;
      for (int k = 0; k < W; ++k) h->st_doff[k] = h->doff[k];
      if (h->fmt == FMT_ELL) {
        h->guard = (int)((g + 1) & ~1LL);
        h->kfmt = FMT_DIA;
      } else {
        for (int k = 0; k < W; ++k) h->doff[k] = 0;  // CSR kernels: column tables
      }
    }
  }

  // ---- device + variant choice -------------------------------------------
  int dev = opt.device;
  if (dev < 0) {
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) {
      delete h;
      return fail(BSOLVE_ERR_CUDA, "cudaGetDevice: %s", cudaGetErrorString(e));
    }
  }
  h->device = dev;
  int prev = -1;
  cudaGetDevice(&prev);
  auto fail_free = [&](int code) {
    free_plan(h);
    if (prev >= 0) cudaSetDevice(prev);
    return code;
  };
  cudaError_t ce = cudaSetDevice(dev);
  if (ce != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_CUDA, "cudaSetDevice(%d): %s", dev, cudaGetErrorString(ce)));
  cudaDeviceProp prop;
  ce = cudaGetDeviceProperties(&prop, dev);
  if (ce != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_CUDA, "cudaGetDeviceProperties: %s", cudaGetErrorString(ce)));
  h->num_sms = prop.multiProcessorCount;
  const int smem_optin = (int)prop.sharedMemPerBlockOptin;
  h->smem_optin = smem_optin;

  // ---- cluster plan: one system per cluster of C CTAs x 1024 rows ---------
  // (DESIGN.md "Kernels" 8).  Auto for 9-point stencils with n > 1024.
  {
    const int rpc = 1024;
    const int c = (n + rpc - 1) / rpc;
    const int last = n - (c - 1) * rpc;
    const bool cl_ok = h->kfmt == FMT_DIA && W == 9 && n > rpc && c <= 8 && n % 2 == 0 &&
                       last >= 1 && h->guard <= rpc &&
                       (opt.block_threads == 0 || opt.block_threads == 128);
    const bool want = opt.placement == BSOLVE_PLACE_CLUSTER ||
                      (opt.placement == BSOLVE_PLACE_AUTO && cl_ok);
    if (want) {
      if (!cl_ok)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                              "cluster placement needs a 9-point stencil (DIA) pattern with even "
                              "1024 < n <= 8192 and stencil reach <= 1024 rows"));
      const int kr = opt.reg_slots ? opt.reg_slots : 4;
      // values in TMEM unless register slots were requested (developer knob
      // BSOLVE_CLUSTER_TMEM=0 selects the register/SMEM-value variant)
      const char *ctenv = getenv("BSOLVE_CLUSTER_TMEM");
      const bool ctmem = opt.reg_slots == 0 && !(ctenv && atoi(ctenv) == 0);
      h->cvar = nullptr;
      // line-tiled TMEM cluster kernel for a 2D grid of a compiled width:
      // opt-in (BSOLVE_CLUSTER_LINE=1), measured 0.88 vs 0.92 M sys/s for the
      // strided-row kernel at n = 4032 (its halo rows are sent by 9 threads
      // with 8 st.async each; 255 registers with spills)
      const char *clenv = getenv("BSOLVE_CLUSTER_LINE");
      const int cl_line = clenv ? atoi(clenv) : 3;  // 3: 3-CTA line kernel, 0: strided rows
      int line_smem = 0;
      // canonical stencil slot -> ELL slot for an NX-wide grid (false: not that grid)
      auto map_c2s = [&](int NX, int (&c2s)[8]) {
        const int canon[8] = {-NX - 1, -NX, -NX + 1, -1, 1, NX - 1, NX, NX + 1};
        for (int cc = 0; cc < 8; ++cc) c2s[cc] = -1;
        for (int k = 1; k < W; ++k) {
          bool real = false;
          for (int rr = 0; rr < n && !real; ++rr) real = h->h_csr2ell[(size_t)k * n + rr] >= 0;
          if (!real) continue;
          const int o = h->doff[k] / 8;
          int cc = 0;
          while (cc < 8 && canon[cc] != o) ++cc;
          if (cc == 8 || c2s[cc] >= 0) return false;
          c2s[cc] = k;
        }
        return true;
      };
      const bool cbj = opt.precond == BSOLVE_PREC_BLOCK_JACOBI;
      if (cbj && !(ctmem && cl_line == 3))
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                              "block-Jacobi on the cluster plan needs the line kernel (TMEM values)"));
      if (ctmem && cl_line == 3) {
        int cnt = 0;
        const CVariant *t = cbj ? variants_cluster_line3_bj(&cnt, &line_smem)
                                : variants_cluster_line3(&cnt, &line_smem);
        const char *csenv = getenv("BSOLVE_CLUSTER_SYNC");  // "barrier": the reference exchange
        // BSOLVE_CLUSTER_SYNC: default / "state": halo state kept per CTA, 2
        // exchanges per iteration, the boundary rows riding the reductions as
        // bulk copies (measured fastest); "halo": bulk halo copies + two-stage
        // reductions, 4 exchanges; "barrier": cluster barriers (the reference)
        const int mb = cbj     ? 1  // block-Jacobi: the halo exchange only
                       : !csenv ? 2
                       : std::strcmp(csenv, "barrier") == 0 ? 0
                       : std::strcmp(csenv, "halo") == 0    ? 1
                                                            : 2;
        for (int i = 0; i < cnt && !h->cvar; ++i) {
          if (t[i].c != c) continue;
          if (t[i].rounds != mb) continue;
          int c2s[8];
          if (!map_c2s(t[i].kreg, c2s)) continue;
          h->cvar = &t[i];
          h->line_nx = t[i].kreg;
          h->line_ctas = 3;
          for (int cc = 0; cc < 8; ++cc) h->c2s[cc] = c2s[cc];
        }
      }
      if (cbj && !h->cvar)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                              "block-Jacobi on the cluster plan needs a 9-point stencil on a "
                              "64-wide grid"));
      if (ctmem && !h->cvar) {
        int cnt = 0;
        const CVariant *t = variants_cluster_tmem(&cnt);
        for (int i = 0; i < cnt; ++i)
          if (t[i].c == c) h->cvar = &t[i];
      } else if (!ctmem) {
        h->cvar = find_cvariant(c, kr, 3);
      }
      if (!h->cvar)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "no cluster variant for C=%d reg_slots=%d",
                              c, kr));
      h->cluster = c;
      h->place = PLACE_CLUSTER;
      h->nt = 128;
      h->r = 8;
      h->n_pad = (n + 1) & ~1;
      h->smem_vals = 9 * rpc;
      // + 4 mbarriers + the TMEM base address slot
      h->smem_bytes = h->line_nx ? line_smem
                                 : (9 * rpc + rpc + 2 * h->guard) * 8 + 16 * c * 4 * 8 + 5 * 8;
      if (h->smem_bytes > smem_optin)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "cluster plan needs %d B of SMEM",
                              h->smem_bytes));
      ce = cudaFuncSetAttribute((const void *)h->cvar->fn,
                                cudaFuncAttributeMaxDynamicSharedMemorySize, h->smem_bytes);
      if (ce != cudaSuccess)
        return fail_free(fail(BSOLVE_ERR_CUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(ce)));
      cudaFuncSetAttribute((const void *)h->cvar->fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                           cudaSharedmemCarveoutMaxShared);
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(c * 64);
      cfg.blockDim = dim3(128);
      cfg.dynamicSmemBytes = h->smem_bytes;
      cudaLaunchAttribute at;
      at.id = cudaLaunchAttributeClusterDimension;
      at.val.clusterDim.x = c;
      at.val.clusterDim.y = 1;
      at.val.clusterDim.z = 1;
      cfg.attrs = &at;
      cfg.numAttrs = 1;
      int ncl = 0;
      ce = cudaOccupancyMaxActiveClusters(&ncl, (const void *)h->cvar->fn, &cfg);
      if (ce != cudaSuccess || ncl < 1)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "cluster of %d CTAs cannot be resident: %s",
                              c, cudaGetErrorString(ce)));
      h->grid_persist = ncl;
      h->max_clusters = ncl;  // (the API's figure; the hardware places CTAs by the limits below)
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&h->occ_api, (const void *)h->cvar->fn, 128,
                                                    h->smem_bytes);
      // resident CTAs per SM from the kernel's own limits, as for the TMEM
      // plan below (registers, SMEM + 1 KB reservation, TMEM columns: the line
      // cluster kernel allocates 128 + 32 per CTA)
      cudaFuncAttributes fa = {};
      if (cudaFuncGetAttributes(&fa, (const void *)h->cvar->fn) == cudaSuccess && fa.numRegs > 0) {
        h->regs = fa.numRegs;
        const int warp_regs = (fa.numRegs * 32 + 255) / 256 * 256;
        const int by_regs = prop.regsPerMultiprocessor / (warp_regs * 4);
        const int by_smem = (int)(prop.sharedMemPerMultiprocessor / (h->smem_bytes + 1024));
        const int by_tmem = h->line_nx ? 512 / 160 : 512 / 128;
        h->ctas_per_sm = std::max(1, std::min(std::min(by_regs, by_smem), by_tmem));
      } else {
        h->ctas_per_sm = std::max(1, (ncl * c + h->num_sms - 1) / h->num_sms);
      }
    }
  }
  // ---- TMEM plan: values in tensor memory (DESIGN.md "Kernels" 9, 10) -----
  // Auto for 9-point stencils up to 1024 rows (measured fastest at n = 992).
  // Line-tiled variant (DESIGN.md "Kernels" 10): the pattern is a 2D 9-point
  // (or 5-point, ...) stencil on an NX-wide grid for a compiled NX, i.e. every
  // slot offset is one of {+-1, +-NX, +-NX+-1}; it is preferred whenever it
  // applies.  Developer knob: BSOLVE_TMEM_LINE=0 keeps the strided kernel.
  const LVariant *line_v = nullptr;
  int line_c2s[8] = {-1, -1, -1, -1, -1, -1, -1, -1};
  int line_width = 0;  // the grid width the chosen line kernel runs
  {
    const char *lenv = getenv("BSOLVE_TMEM_LINE");
    const bool gm = opt.solver == BSOLVE_SOLVER_GMRES;
    const bool bj = opt.precond == BSOLVE_PREC_BLOCK_JACOBI;
    const bool line_on = (gm || !(lenv && atoi(lenv) == 0)) && opt.block_threads == 0 &&
                         opt.reg_slots == 0 && h->st_ok && W <= 9 && n <= 1024 &&
                         h->place != PLACE_CLUSTER &&
                         (opt.placement == BSOLVE_PLACE_AUTO ||
                          opt.placement == BSOLVE_PLACE_TMEM);
    int lcnt = 0;
    const LVariant *lv = line_on ? variants_line(&lcnt) : nullptr;
    // developer knobs: BSOLVE_LINE_CTAS = 2 selects the 2-CTA line kernel
    // (line_kernel.cuh) instead of the 3-CTA one (line3_kernel.cuh);
    // BSOLVE_ROUNDS = reduction rounds per BiCGSTAB iteration (3-CTA default
    // 2 = DESIGN.md R29, 2-CTA default 3)
    const char *ctasenv = getenv("BSOLVE_LINE_CTAS");
    const int lctas = ctasenv ? atoi(ctasenv) : 3;
    const char *roundsenv = getenv("BSOLVE_ROUNDS");
    const int lrounds = roundsenv ? atoi(roundsenv) : (lctas == 3 ? 2 : 3);
    // slot k -> canonical stencil slot of an NX-wide 2D grid (false: not that grid)
    std::vector<char> real_slot(W, 0);  // slot k holds at least one entry of the pattern
    if (line_on)
      for (int k = 1; k < W; ++k)
        for (int r = 0; r < n && !real_slot[k]; ++r)
          real_slot[k] = h->h_csr2ell[(size_t)k * n + r] >= 0;
    auto map_grid = [&](int NX, int (&c2s)[8]) {
      const int canon[8] = {-NX - 1, -NX, -NX + 1, -1, 1, NX - 1, NX, NX + 1};
      for (int c = 0; c < 8; ++c) c2s[c] = -1;
      for (int k = 1; k < W; ++k) {
        if (!real_slot[k]) continue;
        const int o = h->st_doff[k] / 8;
        int c = 0;
        while (c < 8 && canon[c] != o) ++c;
        if (c == 8 || c2s[c] >= 0) return false;
        c2s[c] = k;
      }
      return true;
    };
    // developer knob BSOLVE_LINE_GENERIC=1: the generic-width instance even
    // where a compile-time width exists (tests compare the two bit for bit)
    const char *genv = getenv("BSOLVE_LINE_GENERIC");
    const bool force_generic = genv && atoi(genv) == 1;
    // first pass: the requested geometry; second pass: any 2-CTA variant for the grid
    for (int i = 0; i < 2 * lcnt && !line_v && !force_generic; ++i) {
      const LVariant &cand = lv[i % lcnt];
      if (cand.solver != (gm ? SOLVER_GMRES : SOLVER_BICGSTAB)) continue;
      if (!gm && !bj && cand.rounds != lrounds) continue;
      if (cand.pre != (bj ? 1 : 0)) continue;
      if (bj && i >= lcnt) continue;  // block-Jacobi: the 3-CTA kernel only
      if (i < lcnt) {
        if (!bj && cand.ctas != lctas) continue;
      } else if (cand.ctas != 2) {
        continue;
      }
      int c2s[8];
      if (!map_grid(cand.nx, c2s)) continue;
      line_v = &cand;
      line_width = cand.nx;
      for (int c = 0; c < 8; ++c) line_c2s[c] = c2s[c];
    }
    // generic-width instances (k_line_generic.cu): any width NX = B (mod 8),
    // 3 <= NX <= nxmax (block-Jacobi: NX >= 9, tridiagonal blocks); BiCGSTAB
    // on the 3-CTA kernel, GMRES on the 2-CTA one
    int gcnt = 0;
    const LVariant *gv = (line_on && (gm || bj || (lctas == 3 && lrounds == 2)))
                             ? variants_line_generic(&gcnt) : nullptr;
    for (int nx = bj ? 9 : 3; gv && !line_v && nx <= gv[0].nxmax; ++nx)
      for (int i = 0; i < gcnt && !line_v; ++i) {
        const LVariant &cand = gv[i];
        if (cand.nx != nx % 8 || cand.pre != (bj ? 1 : 0) || nx > cand.nxmax) continue;
        if (cand.solver != (gm ? SOLVER_GMRES : SOLVER_BICGSTAB)) continue;
        int c2s[8];
        if (!map_grid(nx, c2s)) continue;
        line_v = &cand;
        line_width = nx;
        for (int c = 0; c < 8; ++c) line_c2s[c] = c2s[c];
      }
  }
  if (opt.precond == BSOLVE_PREC_BLOCK_JACOBI && !line_v && h->place != PLACE_CLUSTER)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                          "block-Jacobi needs the line-tiled plan: a 2D 9-point stencil on a grid "
                          "of width 9..120 (n <= 1024, placement AUTO or TMEM) or 64 (cluster "
                          "plan, 1024 < n <= 8192)"));
  if (opt.solver == BSOLVE_SOLVER_GMRES && !line_v)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                          "GMRES needs a 2D stencil pattern (9- or 5-point, grid width 3..120) "
                          "with n <= 1024 and placement AUTO or TMEM"));
  const bool tmem_ok = (h->kfmt == FMT_DIA && W == 9 && n <= 1024) || line_v;
  const bool tmem_auto = opt.placement == BSOLVE_PLACE_AUTO && opt.block_threads == 0 &&
                         opt.reg_slots == 0 && tmem_ok;
  if (h->place != PLACE_CLUSTER && (opt.placement == BSOLVE_PLACE_TMEM || tmem_auto)) {
    if (!tmem_ok)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                            "TMEM placement needs a 9-point stencil (DIA) pattern, n <= 1024"));
    h->place = PLACE_TMEM;
    h->n_pad = (n + 1) & ~1;
    h->smem_vals = (int)((h->sys_stride + 1) & ~1LL);
    if (line_v) {
      h->line_nx = line_width;
      h->line_a = line_v->nxmax ? line_width / 8 : 0;
      h->line_generic = line_v->nxmax ? 1 : 0;
      h->var_tmem = line_v->fn;
      h->smem_bytes = line_v->smem_bytes;
      for (int c = 0; c < 8; ++c) h->c2s[c] = line_c2s[c];
      h->nt = 1024 / line_v->r;
      h->r = line_v->r;
      h->line_ctas = line_v->ctas;
    } else {
      // strided TMEM kernel (patterns the line plan does not cover): 128
      // threads x 8 rows, 4 rows per tcgen05.ld wait
      if (opt.block_threads != 0 && opt.block_threads != 128)
        return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "the TMEM plan runs 128 threads per CTA"));
      int tcnt = 0;
      const TVariant *tv = variants_tmem(&tcnt);
      h->var_tmem = tv[0].fn;
      h->nt = tv[0].nt;
      h->r = tv[0].r;
      h->smem_bytes =
          h->smem_vals * 8 + (h->n_pad + 2 * h->guard) * 8 + 16 * (h->nt / 32) * 8 + 16;
    }
    if (h->smem_bytes > smem_optin)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "TMEM plan needs %d B of SMEM", h->smem_bytes));
    ce = cudaFuncSetAttribute((const void *)h->var_tmem,
                              cudaFuncAttributeMaxDynamicSharedMemorySize, h->smem_bytes);
    if (ce != cudaSuccess)
      return fail_free(fail(BSOLVE_ERR_CUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(ce)));
    // the line kernel stages nothing in SMEM (~10 KB per CTA; + the Krylov
    // basis for GMRES): carve out just enough shared memory for 2 CTAs per SM
    // and leave the rest of the unified L1 to the 16-byte value loads
    int carve = (int)cudaSharedmemCarveoutMaxShared;
    if (h->line_nx) {
      const long long need = (long long)h->line_ctas * (h->smem_bytes + 1024);
      carve = (int)std::min<long long>(100, (need * 100 + prop.sharedMemPerMultiprocessor - 1) /
                                                 prop.sharedMemPerMultiprocessor + 5);
    }
    cudaFuncSetAttribute((const void *)h->var_tmem, cudaFuncAttributePreferredSharedMemoryCarveout,
                         carve);
    ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&h->occ_api, h->var_tmem, h->nt,
                                                       h->smem_bytes);
    if (ce != cudaSuccess)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "TMEM variant occupancy query failed"));
    // resident CTAs per SM from the kernel's own limits (registers in 256-
    // register warp units, SMEM incl. the 1 KB per-CTA reservation, threads,
    // TMEM columns: 512 per SM): what ncu reports as launch__occupancy_limit_*
    {
      cudaFuncAttributes fa;
      CUDA_TRY(cudaFuncGetAttributes(&fa, (const void *)h->var_tmem));
      h->regs = fa.numRegs;
      const int warp_regs = (fa.numRegs * 32 + 255) / 256 * 256;
      const int by_regs = prop.regsPerMultiprocessor / (warp_regs * (h->nt / 32));
      const int by_smem = (int)(prop.sharedMemPerMultiprocessor / (h->smem_bytes + 1024));
      const int by_threads = prop.maxThreadsPerMultiProcessor / h->nt;
      const int tcols = h->line_nx ? (h->line_ctas == 3 ? 160 : 128) : 128 * (h->nt / 128);
      const int by_tmem = 512 / tcols;
      h->ctas_per_sm = std::min(std::min(by_regs, by_smem), std::min(by_threads, by_tmem));
    }
    if (h->ctas_per_sm < 1)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "TMEM variant cannot be resident"));
  }
  // rows per thread / CTA size.  Auto: 9-point stencils (DIA) up to 1024 rows
  // take the hybrid 128 threads x 8 rows with 4 off-diagonal slots in
  // registers (measured fastest on B200, DESIGN.md perf log); otherwise 256
  // threads (2 CTAs per SM at <= 128 regs/thread), 512 for 1025..2048 rows.
  if (h->place != PLACE_CLUSTER && h->place != PLACE_TMEM) {
  int nt = opt.block_threads;
  int kreg = opt.reg_slots;
  const bool stencil9 = h->kfmt == FMT_DIA && W == 9 && n <= 1024;
  if (nt == 0) {
    if (stencil9 && (opt.placement == BSOLVE_PLACE_AUTO || opt.placement == BSOLVE_PLACE_SMEM)) {
      nt = 128;
      kreg = 4;
    } else {
      nt = n <= 1024 ? 256 : 512;
    }
  }
  int r = (n + nt - 1) / nt;
  if (r == 3) r = 4;
  if (nt == 512 && r < 4) r = 4;  // the 512-thread variants own 4 rows per thread
  if (nt == 128) {       // hybrid: 8 rows per thread, DIA + SMEM only
    if (n > 1024 || h->kfmt != FMT_DIA || W != 9)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                            "block_threads = 128 needs a 9-slot stencil (DIA) pattern, n <= 1024"));
    r = 8;
  } else if (kreg != 0) {
    return fail_free(fail(BSOLVE_ERR_INVALID, "reg_slots needs block_threads = 128"));
  }
  if (r > 4 && nt != 128)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                          "n = %d needs more than 4 rows per thread at %d threads", n, nt));
  if ((long long)r * nt < n)  // every row must be owned by a thread
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "n = %d exceeds %d threads x %d rows", n, nt, r));
  h->nt = nt;
  h->r = r;
  h->n_pad = (n + 1) & ~1;
  h->smem_vals = (int)((h->sys_stride + 1) & ~1LL);
  const int nwarp = nt / 32;
  const int tail = (h->n_pad + 2 * h->guard) * 8 + 16 * nwarp * 8 + 16;
  const long long smem_need = (long long)h->smem_vals * 8 + tail;
  // PLACE_REGS: persistent kernel, values in registers, staging buffers for
  // values + b + x0 in SMEM (DESIGN.md "Kernels" 7)
  const long long smem_regs = (long long)h->smem_vals * 8 + 2LL * h->n_pad * 8 + tail + 16;
  const bool regs_ok = (h->kfmt == FMT_ELL || h->kfmt == FMT_DIA) && W == 9 && nt == 256 &&
                       n % 2 == 0 && (h->sys_stride * 8) % 16 == 0 && smem_regs <= smem_optin &&
                       find_pvariant(h->kfmt, r) != nullptr;
  int place = opt.placement;
  // AUTO: SMEM-staged values with 2 CTAs per SM measured fastest on B200 for
  // the 992-row workload (DESIGN.md perf log); REGS is opt-in
  if (place == BSOLVE_PLACE_AUTO) place = smem_need <= smem_optin ? PLACE_SMEM : PLACE_STREAM;
  else if (place == BSOLVE_PLACE_REGS) {
    if (!regs_ok)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                            "register-resident placement needs ELL, 9 entries per row, even "
                            "n <= 1024 and %lld B of shared memory",
                            smem_regs));
    place = PLACE_REGS;
  } else
    place = place == BSOLVE_PLACE_SMEM ? PLACE_SMEM : PLACE_STREAM;
  if (place == PLACE_SMEM && smem_need > smem_optin)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED,
                          "SMEM placement needs %lld B of shared memory, device allows %d",
                          smem_need, smem_optin));
  h->place = place;
  // the per-system-CTA kernel: the plan itself (SMEM/STREAM) or the fallback
  // of PLACE_REGS for buffers that are not 16-byte aligned
  const int fb_place = (place == PLACE_STREAM || smem_need > smem_optin) ? PLACE_STREAM : PLACE_SMEM;
  h->smem_bytes_fallback = (int)(fb_place == PLACE_SMEM ? smem_need : tail);
  h->var = find_variant(h->kfmt, fb_place, h->wb, h->wb == 9, r, nt, kreg);
  if (!h->var)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "no kernel variant for fmt=%d place=%d W=%d R=%d NT=%d",
                          h->fmt, fb_place, h->wb, r, nt));
  ce = cudaFuncSetAttribute((const void *)h->var->fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            h->smem_bytes_fallback);
  if (ce != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_CUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(ce)));
  cudaFuncSetAttribute((const void *)h->var->fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                       cudaSharedmemCarveoutMaxShared);
  if (place == PLACE_REGS) {
    h->pvar = find_pvariant(h->kfmt, r);
    h->smem_bytes = (int)smem_regs;
    ce = cudaFuncSetAttribute((const void *)h->pvar->fn,
                              cudaFuncAttributeMaxDynamicSharedMemorySize, h->smem_bytes);
    if (ce != cudaSuccess)
      return fail_free(fail(BSOLVE_ERR_CUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(ce)));
    ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&h->ctas_per_sm, h->pvar->fn, nt,
                                                       h->smem_bytes);
    if (cudaMalloc(&h->d_ctr, 2 * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMemset(h->d_ctr, 0, 2 * sizeof(unsigned long long)) != cudaSuccess)
      return fail_free(fail(BSOLVE_ERR_NOMEM, "work counter allocation failed"));
  } else {
    h->smem_bytes = h->smem_bytes_fallback;
    ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&h->ctas_per_sm, h->var->fn, nt,
                                                       h->smem_bytes);
  }
  if (ce != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_CUDA, "occupancy query: %s", cudaGetErrorString(ce)));
  if (h->ctas_per_sm < 1)
    return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "kernel variant cannot be resident on an SM"));
  h->grid_persist = h->num_sms * h->ctas_per_sm;
  }  // single-CTA plans

  // ---- device copy of the pattern ------------------------------------------
  std::vector<int32_t> rp(row_ptr, row_ptr + n + 1);
  const size_t ell_b = sizeof(int32_t) * (size_t)W * n;
  // Column table the kernels read, [W][n]: ELL -> the slot map; CSR -> the
  // k-th CSR entry of each row (padding: own row, never multiplied).
  std::vector<int32_t> kcols = h->h_ell_col;
  if (h->fmt == FMT_CSR)
    for (int i = 0; i < n; ++i)
      for (int k = 0; k < W; ++k) {
        const int e = row_ptr[i] + k;
        kcols[(size_t)k * n + i] = e < row_ptr[i + 1] ? col_idx[e] : i;
      }
  if (cudaMalloc(&h->d_ell_col, ell_b) != cudaSuccess ||
      cudaMalloc(&h->d_src, ell_b) != cudaSuccess ||
      cudaMalloc(&h->d_row_ptr, sizeof(int32_t) * (n + 1)) != cudaSuccess ||
      cudaMalloc(&h->d_diag, sizeof(int32_t) * n) != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_NOMEM, "device allocation of the pattern failed"));
  if (cudaMemcpy(h->d_ell_col, kcols.data(), ell_b, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(h->d_src, h->h_csr2ell.data(), ell_b, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(h->d_row_ptr, rp.data(), sizeof(int32_t) * (n + 1), cudaMemcpyHostToDevice) !=
          cudaSuccess ||
      cudaMemcpy(h->d_diag, diag.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice) != cudaSuccess)
    return fail_free(fail(BSOLVE_ERR_CUDA, "copy of the pattern to the device failed"));
  if (h->line_nx && h->fmt == FMT_CSR && h->place == PLACE_TMEM) {
    // CSR values on the line-tiled plan: where each (row, canonical slot)
    // value sits inside a system's CSR block (the ELL slot map's source index)
    std::vector<int32_t> vidx((size_t)9 * n, -1);
    for (int c = 0; c < 8; ++c)
      if (h->c2s[c] >= 0)
        for (int r = 0; r < n; ++r) vidx[(size_t)c * n + r] = h->h_csr2ell[(size_t)h->c2s[c] * n + r];
    for (int r = 0; r < n; ++r) vidx[(size_t)8 * n + r] = h->h_csr2ell[r];  // slot 0: diagonal
    if (cudaMalloc(&h->d_vidx, sizeof(int32_t) * vidx.size()) != cudaSuccess ||
        cudaMemcpy(h->d_vidx, vidx.data(), sizeof(int32_t) * vidx.size(), cudaMemcpyHostToDevice) !=
            cudaSuccess)
      return fail_free(fail(BSOLVE_ERR_CUDA, "copy of the CSR value index table failed"));
  }
  if (h->direct_fallback) {
    // banded tables + fallback buffers now, so bsolve_run never allocates:
    // the fused banded kernel on at most one wave of resident CTAs, its
    // workspace capped at 256 MB (failures are rare; the grid bounds memory)
    int rc = setup_banded(h);
    if (rc) return fail_free(rc);
    int occ = 0;
    ce = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, (const void *)h->bvar->fn,
                                                       h->bvar->nt, h->bvar->smem_bytes);
    if (ce != cudaSuccess || occ < 1)
      return fail_free(fail(BSOLVE_ERR_UNSUPPORTED, "direct_fallback: banded kernel cannot be resident"));
    const long long cap = std::max<long long>(1, (256ll << 20) / (16ll * (long long)banded_ws_sys(h)));
    h->fb_grid = (int)std::min<long long>((long long)occ * h->num_sms, cap);
    rc = alloc_fallback(h, h->fb_grid, batch, &h->d_fbws, &h->d_fbl, &h->d_fbn);
    if (rc) return fail_free(rc);
  }
  if (prev >= 0) cudaSetDevice(prev);
  *out = h;
  return BSOLVE_OK;
}

extern "C" int bsolve_destroy(bsolve_handle h) {
  free_plan(h);
  return BSOLVE_OK;
}

extern "C" const char *bsolve_last_error(void) { return g_err.c_str(); }

extern "C" int bsolve_query(bsolve_handle h, bsolve_info *info) {
  if (!h || !info) return fail(BSOLVE_ERR_INVALID, "NULL handle or info");
  info->n = h->n;
  info->nnz = h->nnz;
  info->batch = h->batch;
  info->ell_width = h->W;
  info->format = h->fmt == FMT_ELL ? BSOLVE_FMT_ELL : BSOLVE_FMT_CSR;
  info->placement = h->place == PLACE_SMEM ? BSOLVE_PLACE_SMEM
                    : h->place == PLACE_REGS    ? BSOLVE_PLACE_REGS
                    : h->place == PLACE_CLUSTER ? BSOLVE_PLACE_CLUSTER
                    : h->place == PLACE_TMEM    ? BSOLVE_PLACE_TMEM
                                                : BSOLVE_PLACE_STREAM;
  info->block_threads = h->nt;
  info->rows_per_thread = h->r;
  info->smem_bytes = h->smem_bytes;
  info->ctas_per_sm = h->ctas_per_sm;
  info->regs_per_thread = h->regs;
  info->occupancy_api = h->occ_api;
  info->line_width = h->line_nx;
  info->line_generic = h->line_generic;
  info->max_active_clusters = h->max_clusters;
  info->num_sms = h->num_sms;
  info->grid = h->place == PLACE_REGS      ? (int)std::min<long long>(h->grid_persist, h->batch)
               : h->place == PLACE_CLUSTER ? h->batch * h->cluster
                                           : h->batch;
  info->cluster = h->cluster;
  info->kl = h->kl;
  info->ku = h->ku;
  info->device = h->device;
  info->kernel_mode = h->line_nx ? 4 : h->kfmt;
  info->solver = h->solver;
  info->precond = h->precond;
  info->restart = h->restart;
  info->banded_launches = h->banded_launches;
  return BSOLVE_OK;
}

extern "C" int bsolve_ell_map(bsolve_handle h, int32_t *cols, int32_t *src) {
  if (!h || (!cols && !src)) return fail(BSOLVE_ERR_INVALID, "NULL handle or outputs");
  if (cols) std::memcpy(cols, h->h_ell_col.data(), sizeof(int32_t) * h->h_ell_col.size());
  if (src) std::memcpy(src, h->h_csr2ell.data(), sizeof(int32_t) * h->h_csr2ell.size());
  return BSOLVE_OK;
}

// ------------------------------------------------------------------ run --
static int check_run_args(bsolve_handle h, const double *values, const double *b, double tol,
                          int maxiter, const double *x, const int32_t *iters,
                          const double *resnorm) {
  if (!h) return fail(BSOLVE_ERR_INVALID, "handle is NULL");
  if (h->batch > 0 && (!values || !b || !x || !iters || !resnorm))
    return fail(BSOLVE_ERR_INVALID, "values, b, x, iters and resnorm must be non-NULL");
  if (!(tol >= 0.0) || !std::isfinite(tol))
    return fail(BSOLVE_ERR_INVALID, "tol = %g must be finite and >= 0", tol);
  if (maxiter < 0) return fail(BSOLVE_ERR_INVALID, "maxiter = %d must be >= 0", maxiter);
  return BSOLVE_OK;
}

static int launch_fallback(bsolve_handle h, const double *values, const double *b, double *x,
                           int8_t *status, double *resnorm, long long count, cudaStream_t stream,
                           int slot);
static int launch_banded(bsolve_handle h, const double *values, const double *b, double *x,
                         int32_t *info, int32_t *ipiv, long long count, cudaStream_t stream,
                         int slot = -1);

static int launch_solve(bsolve_handle h, const double *values, const double *b, const double *x0,
                        double tol, int maxiter, double *x, int32_t *iters, double *resnorm,
                        int8_t *status, int count, cudaStream_t stream, int slot = -1) {
  if (count <= 0) return BSOLVE_OK;
  SolveParams P = {};
  P.values = values;
  P.b = b;
  P.x0 = x0;
  P.x = x;
  P.iters = iters;
  P.resnorm = resnorm;
  P.status = status;
  P.ell_col = h->d_ell_col;
  P.row_ptr = h->d_row_ptr;
  P.diag_slot = h->d_diag;
  P.sys_stride = h->sys_stride;
  P.tol = tol;
  P.n = h->n;
  P.W = h->W;
  P.batch = count;
  P.maxiter = maxiter;
  P.stop = h->stop;
  P.trc = h->trc;
  P.smem_vals = h->smem_vals;
  P.n_pad = h->n_pad;
  P.guard = h->guard;
  for (int k = 0; k < kMaxW; ++k) P.doff[k] = h->doff[k];
  for (int c = 0; c < 8; ++c) P.c2s[c] = h->c2s[c];
  P.vidx = h->d_vidx;
  P.precond = h->precond;
  P.restart = h->restart;
  // line plan: each CTA asks L2 for the system that will start about one
  // residency later (CTAs dispatch in blockIdx order, 2 per SM), so its
  // start-up loads hit L2 instead of HBM (BSOLVE_L2_PREFETCH=0 disables)
  {
    const char *pe = getenv("BSOLVE_L2_PREFETCH");
    // systems ahead, in units of #SMs (cluster plan: off, measured 1.29 vs 1.27 M sys/s at n = 4032)
    const int k = pe ? atoi(pe) : (h->place == PLACE_CLUSTER ? 0 : 2);
    P.pf_ahead = (h->line_nx && k > 0) ? k * h->num_sms : 0;
    P.line_a = h->line_a;
  }
  const bool aligned = ((reinterpret_cast<uintptr_t>(values) | reinterpret_cast<uintptr_t>(b) |
                         reinterpret_cast<uintptr_t>(x0)) & 15u) == 0;
  if (h->place == PLACE_TMEM) {  // (unaligned values: the kernel copies without TMA)
    h->var_tmem<<<count, h->nt, h->smem_bytes, stream>>>(P);
  } else if (h->place == PLACE_CLUSTER) {
    if ((reinterpret_cast<uintptr_t>(values) & 15u) != 0)
      return fail(BSOLVE_ERR_INVALID, "the cluster plan needs 16-byte aligned values (TMA)");
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)count * (unsigned)h->cluster);
    cfg.blockDim = dim3(h->nt);
    cfg.dynamicSmemBytes = h->smem_bytes;
    cfg.stream = stream;
    cudaLaunchAttribute at;
    at.id = cudaLaunchAttributeClusterDimension;
    at.val.clusterDim.x = h->cluster;
    at.val.clusterDim.y = 1;
    at.val.clusterDim.z = 1;
    cfg.attrs = &at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, h->cvar->fn, P);
    if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "cluster launch: %s", cudaGetErrorString(e));
  } else if (h->place == PLACE_REGS && aligned) {
    const int grid = (int)std::min<long long>(h->grid_persist, count);
    h->pvar->fn<<<grid, h->nt, h->smem_bytes, stream>>>(P, h->d_ctr);
  } else {
    h->var->fn<<<count, h->nt, h->smem_bytes_fallback, stream>>>(P);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "solve launch: %s", cudaGetErrorString(e));
  if (h->direct_fallback)  // non-converged systems -> banded LU
    return launch_fallback(h, values, b, x, status, resnorm, count, stream, slot);
  return BSOLVE_OK;
}

static int check_device_ptr(bsolve_handle h, const void *p, const char *name) {
  if (!p) return BSOLVE_OK;
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(BSOLVE_ERR_INVALID, "%s is not a CUDA pointer (%s)", name, cudaGetErrorString(e));
  }
  if (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged)
    return fail(BSOLVE_ERR_INVALID, "%s must be device memory", name);
  if (a.type == cudaMemoryTypeDevice && a.device != h->device)
    return fail(BSOLVE_ERR_INVALID, "%s lives on device %d, handle is on device %d", name, a.device,
                h->device);
  return BSOLVE_OK;
}

extern "C" int bsolve_run(bsolve_handle h, const double *values, const double *b, const double *x0,
                          double tol, int maxiter, double *x, int32_t *iters, double *resnorm,
                          int8_t *status, void *stream) {
  g_err.clear();
  int rc = check_run_args(h, values, b, tol, maxiter, x, iters, resnorm);
  if (rc) return rc;
  if (h->batch == 0) return BSOLVE_OK;
  if (h->direct_fallback && !status)
    return fail(BSOLVE_ERR_INVALID, "direct_fallback needs the status array (it selects the "
                                    "systems the banded solver re-solves)");
  const void *ptrs[] = {values, b, x0, x, iters, resnorm, status};
  const char *names[] = {"values", "b", "x0", "x", "iters", "resnorm", "status"};
  for (int i = 0; i < 7; ++i)
    if ((rc = check_device_ptr(h, ptrs[i], names[i]))) return rc;
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  rc = launch_solve(h, values, b, x0, tol, maxiter, x, iters, resnorm, status, h->batch,
                    (cudaStream_t)stream);
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  return rc;
}

// Lazily set up the host-buffer pipeline (bsolve_run_host,
// bsolve_banded_solve_host): 3 non-blocking streams, each with device
// buffers for one chunk of ~64 MB of values (whole waves of resident CTAs).
static int ensure_host_pipeline(bsolve_handle h) {
  if (h->h_chunk != 0) return BSOLVE_OK;
  const int n = h->n;
  const long long ss = h->sys_stride;
  const long long wave = (long long)h->num_sms * h->ctas_per_sm;
  long long c = std::max<long long>(wave, (64ll << 20) / (ss * 8));
  c = (c + wave - 1) / wave * wave;
  c = std::min<long long>(c, h->batch);
  const int chunk = (int)std::max<long long>(c, 1);
  for (int s = 0; s < bsolve_plan::kSlots; ++s) {
    CUDA_TRY(cudaStreamCreateWithFlags(&h->hs[s], cudaStreamNonBlocking));
    const size_t c_ = (size_t)chunk;
    if (cudaMalloc(&h->h_val[s], c_ * ss * 8) != cudaSuccess ||
        cudaMalloc(&h->h_b[s], c_ * n * 8) != cudaSuccess ||
        cudaMalloc(&h->h_x0[s], c_ * n * 8) != cudaSuccess ||
        cudaMalloc(&h->h_x[s], c_ * n * 8) != cudaSuccess ||
        cudaMalloc(&h->h_res[s], c_ * 8) != cudaSuccess ||
        cudaMalloc(&h->h_it[s], c_ * 4) != cudaSuccess ||
        cudaMalloc(&h->h_st[s], c_) != cudaSuccess) {
      cudaGetLastError();
      return fail(BSOLVE_ERR_NOMEM, "device allocation for the host pipeline failed");
    }
    if (h->direct_fallback) {  // each slot's stream runs its own fallback (smaller grid)
      const int rc = alloc_fallback(h, std::max(1, h->fb_grid / bsolve_plan::kSlots), chunk,
                                    &h->h_fbws[s], &h->h_fbl[s], &h->h_fbn[s]);
      if (rc) return rc;
    }
  }
  h->h_chunk = chunk;
  return BSOLVE_OK;
}

extern "C" int bsolve_run_host(bsolve_handle h, const double *values, const double *b,
                               const double *x0, double tol, int maxiter, double *x, int32_t *iters,
                               double *resnorm, int8_t *status) {
  g_err.clear();
  int rc = check_run_args(h, values, b, tol, maxiter, x, iters, resnorm);
  if (rc) return rc;
  if (h->batch == 0) return BSOLVE_OK;
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  const int n = h->n;
  const long long ss = h->sys_stride;
  if ((rc = ensure_host_pipeline(h))) return rc;
  const int C = h->h_chunk;
  int k = 0;
  for (long long s0 = 0; s0 < h->batch; s0 += C, ++k) {
    const int cnt = (int)std::min<long long>(C, h->batch - s0);
    const int sl = k % bsolve_plan::kSlots;
    cudaStream_t st = h->hs[sl];
    CUDA_TRY(cudaMemcpyAsync(h->h_val[sl], values + s0 * ss, (size_t)cnt * ss * 8,
                             cudaMemcpyHostToDevice, st));
    CUDA_TRY(cudaMemcpyAsync(h->h_b[sl], b + s0 * n, (size_t)cnt * n * 8, cudaMemcpyHostToDevice, st));
    if (x0)
      CUDA_TRY(cudaMemcpyAsync(h->h_x0[sl], x0 + s0 * n, (size_t)cnt * n * 8,
                               cudaMemcpyHostToDevice, st));
    rc = launch_solve(h, h->h_val[sl], h->h_b[sl], x0 ? h->h_x0[sl] : nullptr, tol, maxiter,
                      h->h_x[sl], h->h_it[sl], h->h_res[sl], h->h_st[sl], cnt, st, sl);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(x + s0 * n, h->h_x[sl], (size_t)cnt * n * 8, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaMemcpyAsync(iters + s0, h->h_it[sl], (size_t)cnt * 4, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaMemcpyAsync(resnorm + s0, h->h_res[sl], (size_t)cnt * 8, cudaMemcpyDeviceToHost, st));
    if (status)
      CUDA_TRY(cudaMemcpyAsync(status + s0, h->h_st[sl], (size_t)cnt, cudaMemcpyDeviceToHost, st));
  }
  for (int s = 0; s < bsolve_plan::kSlots; ++s) CUDA_TRY(cudaStreamSynchronize(h->hs[s]));
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  return BSOLVE_OK;
}

extern "C" int bsolve_spmv(bsolve_handle h, const double *values, const double *x, double *y,
                           int batch, void *stream) {
  g_err.clear();
  if (!h) return fail(BSOLVE_ERR_INVALID, "handle is NULL");
  if (batch < 0) return fail(BSOLVE_ERR_INVALID, "batch = %d must be >= 0", batch);
  if (batch == 0) return BSOLVE_OK;
  if (!values || !x || !y) return fail(BSOLVE_ERR_INVALID, "values, x and y must be non-NULL");
  if (x == y) return fail(BSOLVE_ERR_INVALID, "y must not alias x");
  int rc;
  const void *ptrs[] = {values, x, y};
  const char *names[] = {"values", "x", "y"};
  for (int i = 0; i < 3; ++i)
    if ((rc = check_device_ptr(h, ptrs[i], names[i]))) return rc;
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  const size_t sm = sizeof(double) * h->n;
  if (h->fmt == FMT_ELL) {
    if (sm > 48 * 1024)
      CUDA_TRY(cudaFuncSetAttribute((const void *)spmv_kernel<FMT_ELL, 256>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    spmv_kernel<FMT_ELL, 256><<<batch, 256, sm, (cudaStream_t)stream>>>(
        values, x, y, h->d_ell_col, h->d_row_ptr, h->n, h->W, h->sys_stride);
  } else {
    if (sm > 48 * 1024)
      CUDA_TRY(cudaFuncSetAttribute((const void *)spmv_kernel<FMT_CSR, 256>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    spmv_kernel<FMT_CSR, 256><<<batch, 256, sm, (cudaStream_t)stream>>>(
        values, x, y, h->d_ell_col, h->d_row_ptr, h->n, h->W, h->sys_stride);
  }
  cudaError_t e = cudaGetLastError();
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "spmv launch: %s", cudaGetErrorString(e));
  return BSOLVE_OK;
}

extern "C" int bsolve_csr_to_ell(bsolve_handle h, const double *csr_values, double *ell_values,
                                 int batch, void *stream) {
  g_err.clear();
  if (!h) return fail(BSOLVE_ERR_INVALID, "handle is NULL");
  if (batch < 0) return fail(BSOLVE_ERR_INVALID, "batch = %d must be >= 0", batch);
  if (batch == 0) return BSOLVE_OK;
  if (!csr_values || !ell_values) return fail(BSOLVE_ERR_INVALID, "NULL values");
  int rc;
  if ((rc = check_device_ptr(h, csr_values, "csr_values"))) return rc;
  if ((rc = check_device_ptr(h, ell_values, "ell_values"))) return rc;
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  const long long slots = (long long)h->W * h->n;
  const long long total = slots * batch;
  const int blocks = (int)std::min<long long>((total + 255) / 256, (long long)h->num_sms * 16);
  csr_to_ell_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(csr_values, ell_values, h->d_src,
                                                               slots, h->nnz, total);
  cudaError_t e = cudaGetLastError();
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "csr_to_ell launch: %s", cudaGetErrorString(e));
  return BSOLVE_OK;
}

// ---------------------------------------------- banded direct solver (f4) --
// Pick the banded instance that covers the pattern and upload its tables
// (pattern entry -> value index + ring position; the ELL column of every
// slot for the fallback's residual).  Synchronous host work: bsolve_create
// runs it when direct_fallback is set, bsolve_banded_solve on its first call.
static int setup_banded(bsolve_handle h) {
  if (h->bvar) return BSOLVE_OK;
  const int kb = std::max(h->kl, h->ku);
  int cnt = 0;
  const BVariant *tab = variants_banded(&cnt), *bv = nullptr;
  for (int i = 0; i < cnt; ++i)  // smallest padded bandwidth that covers the pattern
    if (tab[i].kb >= kb && tab[i].max_entries > h->W && (!bv || tab[i].kb < bv->kb)) bv = &tab[i];
  if (!bv)
    return fail(BSOLVE_ERR_UNSUPPORTED,
                "banded solver: bandwidth kl = %d, ku = %d exceeds the largest instance", h->kl,
                h->ku);
  if ((long long)h->sys_stride >= (1LL << 23))
    return fail(BSOLVE_ERR_UNSUPPORTED, "banded solver: %lld values per system exceed 2^23",
                h->sys_stride);
  const int n = h->n, W = h->W;
  const int Wb = 2 * bv->kb + 1;  // the instance's window width
  // entry k of row r: its value index inside one system's block (CSR order
  // or ELL slot k) and the ring position (column mod Wb); padding -> -1
  std::vector<int32_t> bnd((size_t)W * n, -1);
  for (int k = 0; k < W; ++k)
    for (int r = 0; r < n; ++r) {
      const int e = h->h_csr2ell[(size_t)k * n + r];
      if (e < 0) continue;
      const long long vidx = h->fmt == FMT_ELL ? (long long)k * n + r : e;
      const int col = h->h_ell_col[(size_t)k * n + r];
      bnd[(size_t)k * n + r] = (int32_t)((vidx << 8) | (col % Wb));
    }
  const size_t tb = sizeof(int32_t) * bnd.size();
  if (cudaMalloc(&h->d_bnd, tb) != cudaSuccess || cudaMalloc(&h->d_bcol, tb) != cudaSuccess) {
    cudaGetLastError();
    return fail(BSOLVE_ERR_NOMEM, "banded solver: pattern table allocation failed");
  }
  if (cudaMemcpy(h->d_bnd, bnd.data(), tb, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(h->d_bcol, h->h_ell_col.data(), tb, cudaMemcpyHostToDevice) != cudaSuccess)
    return fail(BSOLVE_ERR_CUDA, "banded solver: pattern table copy failed");
  if (bv->smem_bytes > 48 * 1024) {
    CUDA_TRY(cudaFuncSetAttribute((const void *)bv->fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  bv->smem_bytes));
    CUDA_TRY(cudaFuncSetAttribute((const void *)bv->fn_split,
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, bv->smem_bytes));
  }
  h->bnd_w = Wb;
  h->bvar = bv;
  return BSOLVE_OK;
}

static size_t banded_ws_sys(bsolve_handle h) {  // doubles of U + y per system
  return (size_t)h->n * h->bnd_w + h->n;
}

// Direct fallback buffers (the fused kernel's double-buffered per-CTA
// workspace for `grid` CTAs, the compacted list, its length).
static int alloc_fallback(bsolve_handle h, int grid, long long list_len, double **ws,
                          int32_t **list, int32_t **len) {
  if (cudaMalloc(ws, sizeof(double) * (size_t)grid * 2 * banded_ws_sys(h)) != cudaSuccess ||
      cudaMalloc(list, sizeof(int32_t) * (size_t)std::max<long long>(1, list_len)) != cudaSuccess ||
      cudaMalloc(len, sizeof(int32_t)) != cudaSuccess) {
    cudaGetLastError();
    return fail(BSOLVE_ERR_NOMEM, "direct_fallback: workspace allocation failed");
  }
  return BSOLVE_OK;
}

// direct_fallback (R27): after the iterative launch, list the
// systems whose status is not CONVERGED on the device, then ONE fused banded
// launch (factor warps + back-substitution warp, per-CTA double-buffered
// workspace) solves only those.  No allocation, no host synchronisation:
// 3 asynchronous operations (memset of the counter, compaction, solve); with
// no failed system the solve kernel exits at once.
static int launch_fallback(bsolve_handle h, const double *values, const double *b, double *x,
                           int8_t *status, double *resnorm, long long count, cudaStream_t stream,
                           int slot) {
  const BVariant *bv = h->bvar;
  double *ws = slot >= 0 ? h->h_fbws[slot] : h->d_fbws;
  int32_t *list = slot >= 0 ? h->h_fbl[slot] : h->d_fbl;
  int32_t *len = slot >= 0 ? h->h_fbn[slot] : h->d_fbn;
  if (!bv || !ws || !list || !len)
    return fail(BSOLVE_ERR_INVALID, "direct_fallback buffers are missing (handle not set up)");
  CUDA_TRY(cudaMemsetAsync(len, 0, sizeof(int32_t), stream));
  const int cgrid = (int)std::min<long long>((count + 255) / 256, (long long)h->num_sms * 4);
  bband::fallback_compact_kernel<<<cgrid, 256, 0, stream>>>(status, count, list, len);
  bband::BandParams P;
  P.values = values;
  P.b = b;
  P.bnd = h->d_bnd;
  P.cols = h->d_bcol;
  P.x = x;
  P.info = nullptr;
  P.ipiv = nullptr;
  P.only = status;
  P.resnorm = resnorm;
  P.ws = ws;
  P.list = list;
  P.list_len = len;
  P.sys_stride = h->sys_stride;
  P.E = h->W;
  P.n = h->n;
  P.batch = (int)count;
  const int grid = slot >= 0 ? std::max(1, h->fb_grid / bsolve_plan::kSlots) : h->fb_grid;
  bv->fn<<<grid, bv->nt, bv->smem_bytes, stream>>>(P);
  h->banded_launches = 2;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "fallback launch: %s", cudaGetErrorString(e));
  return BSOLVE_OK;
}

// Standalone banded solve of `count` systems (bsolve_banded_solve[_host]).
// Split mode (default; BSOLVE_BANDED_SPLIT=0 selects the fused kernel):
// factor-only CTAs (more per SM) write U, y per system into a chunk
// workspace, then one warp per system back-substitutes; chunks of systems
// keep the workspace bounded.
static int launch_banded(bsolve_handle h, const double *values, const double *b, double *x,
                         int32_t *info, int32_t *ipiv, long long count, cudaStream_t stream,
                         int slot) {
  if (count <= 0) return BSOLVE_OK;
  int rc = setup_banded(h);
  if (rc) return rc;
  const BVariant *bv = h->bvar;
  const int n = h->n;
  const int Wb = h->bnd_w;
  bband::BandParams P;
  P.values = values;
  P.b = b;
  P.bnd = h->d_bnd;
  P.cols = h->d_bcol;
  P.x = x;
  P.info = info;
  P.ipiv = ipiv;
  P.only = nullptr;
  P.resnorm = nullptr;
  P.list = nullptr;
  P.list_len = nullptr;
  P.sys_stride = h->sys_stride;
  P.E = h->W;
  P.n = n;
  const size_t ws_sys = banded_ws_sys(h);
  // the back substitution keeps x of each of its warps in SMEM: as many
  // warps per CTA (<= 4) as the device's SMEM allows, else the fused kernel
  const int bs_warps =
      (int)std::min<long long>(4, (long long)h->smem_optin / ((long long)(n + Wb) * 8));
  const char *senv = getenv("BSOLVE_BANDED_SPLIT");
  const bool split = !(senv && atoi(senv) == 0) && bs_warps >= 1;
  // split mode factorisation: one warp per system (banded_lu_warp_kernel) when
  // the instance has one and a row's entries + b fit the 32 loader lanes;
  // developer knob BSOLVE_BANDED_WARP=0 keeps the multi-warp CTA kernel
  const char *wenv = getenv("BSOLVE_BANDED_WARP");
  const bool warp = split && bv->fn_warp && h->W + 1 <= 32 && !(wenv && atoi(wenv) == 0);
  banded_fn fact = warp ? bv->fn_warp : split ? bv->fn_split : bv->fn;
  const int nt = warp ? 32 : split ? bv->nt_split : bv->nt;
  const int fsmem = warp ? bv->smem_warp : bv->smem_bytes;
  if (warp)
    cudaFuncSetAttribute((const void *)fact, cudaFuncAttributePreferredSharedMemoryCarveout,
                         cudaSharedmemCarveoutMaxShared);
  int occ = 0;
  CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, (const void *)fact, nt, fsmem));
  if (occ < 1) return fail(BSOLVE_ERR_UNSUPPORTED, "banded kernel cannot be resident");
  const long long resident = (long long)occ * h->num_sms;
  long long chunk = count;
  size_t need;
  if (split) {
    // at most ~8 GB of workspace, at least one full wave of CTAs
    // (a whole number of resident-CTA waves: no partial last wave per chunk)
    chunk = std::max<long long>(1, (long long)((8ull << 30) / (8 * ws_sys)) / resident) * resident;
    chunk = std::min<long long>(chunk, count);
    need = sizeof(double) * (size_t)chunk * ws_sys;
  } else {
    need = sizeof(double) * (size_t)std::min<long long>(resident, count) * 2 * ws_sys;
  }
  // workspace: the handle's, or host-pipeline slot `slot`'s (concurrent streams)
  double *&wsp = slot >= 0 ? h->h_bws[slot] : h->d_bws;
  size_t &wsb = slot >= 0 ? h->h_bws_bytes[slot] : h->bws_bytes;
  if (wsb < need) {
    cudaFree(wsp);
    wsp = nullptr;
    wsb = 0;
    if (cudaMalloc(&wsp, need) != cudaSuccess) {
      cudaGetLastError();
      return fail(BSOLVE_ERR_NOMEM, "banded solver: %zu B workspace allocation failed", need);
    }
    wsb = need;
  }
  P.ws = wsp;
  h->banded_launches = split ? (int)(2 * ((count + chunk - 1) / chunk)) : 1;
  if (!split) {
    P.batch = count;
    const int grid = (int)std::min<long long>(resident, count);
    fact<<<grid, nt, bv->smem_bytes, stream>>>(P);
  } else {
    const int sbs = bs_warps * (n + Wb) * (int)sizeof(double);  // per-warp x arrays
    if (sbs > 48 * 1024)
      CUDA_TRY(cudaFuncSetAttribute((const void *)bv->fn_backsub,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, sbs));
    for (long long c0 = 0; c0 < count; c0 += chunk) {
      const long long cnt = std::min<long long>(chunk, count - c0);
      bband::BandParams Q = P;
      Q.values = values + c0 * h->sys_stride;
      Q.b = b + c0 * n;
      Q.x = x + c0 * n;
      Q.info = info ? info + c0 : nullptr;
      Q.ipiv = ipiv ? ipiv + c0 * n : nullptr;
      Q.batch = cnt;
      fact<<<(int)std::min<long long>(resident, cnt), nt, fsmem, stream>>>(Q);
      const int gb =
          (int)std::min<long long>((cnt + bs_warps - 1) / bs_warps, (long long)h->num_sms * 16);
      bv->fn_backsub<<<gb, 32 * bs_warps, sbs, stream>>>(Q);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "banded launch: %s", cudaGetErrorString(e));
  return BSOLVE_OK;
}

extern "C" int bsolve_banded_solve(bsolve_handle h, const double *values, const double *b,
                                   double *x, int32_t *info, int32_t *ipiv, void *stream) {
  g_err.clear();
  if (!h) return fail(BSOLVE_ERR_INVALID, "handle is NULL");
  if (h->batch == 0) return BSOLVE_OK;
  if (!values || !b || !x || !info)
    return fail(BSOLVE_ERR_INVALID, "values, b, x and info must be non-NULL");
  int rc;
  const void *ptrs[] = {values, b, x, info, ipiv};
  const char *names[] = {"values", "b", "x", "info", "ipiv"};
  for (int i = 0; i < 5; ++i)
    if ((rc = check_device_ptr(h, ptrs[i], names[i]))) return rc;
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  rc = launch_banded(h, values, b, x, info, ipiv, h->batch, (cudaStream_t)stream);
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  return rc;
}

extern "C" int bsolve_banded_solve_host(bsolve_handle h, const double *values, const double *b,
                                        double *x, int32_t *info) {
  g_err.clear();
  if (!h) return fail(BSOLVE_ERR_INVALID, "handle is NULL");
  if (h->batch == 0) return BSOLVE_OK;
  if (!values || !b || !x || !info)
    return fail(BSOLVE_ERR_INVALID, "values, b, x and info must be non-NULL");
  int prev = -1;
  cudaGetDevice(&prev);
  if (prev != h->device) CUDA_TRY(cudaSetDevice(h->device));
  int rc = ensure_host_pipeline(h);
  if (rc) return rc;
  const int n = h->n;
  const long long ss = h->sys_stride;
  const int C = h->h_chunk;
  int k = 0;
  for (long long s0 = 0; s0 < h->batch; s0 += C, ++k) {
    const int cnt = (int)std::min<long long>(C, h->batch - s0);
    const int sl = k % bsolve_plan::kSlots;
    cudaStream_t st = h->hs[sl];
    CUDA_TRY(cudaMemcpyAsync(h->h_val[sl], values + s0 * ss, (size_t)cnt * ss * 8,
                             cudaMemcpyHostToDevice, st));
    CUDA_TRY(cudaMemcpyAsync(h->h_b[sl], b + s0 * n, (size_t)cnt * n * 8, cudaMemcpyHostToDevice, st));
    rc = launch_banded(h, h->h_val[sl], h->h_b[sl], h->h_x[sl], h->h_it[sl], nullptr, cnt, st, sl);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(x + s0 * n, h->h_x[sl], (size_t)cnt * n * 8, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaMemcpyAsync(info + s0, h->h_it[sl], (size_t)cnt * 4, cudaMemcpyDeviceToHost, st));
  }
  for (int s = 0; s < bsolve_plan::kSlots; ++s) CUDA_TRY(cudaStreamSynchronize(h->hs[s]));
  if (prev >= 0 && prev != h->device) cudaSetDevice(prev);
  return BSOLVE_OK;
}

extern "C" int bsolve_probe_smem_bandwidth(int device, double *bytes_per_s, double *sm_hz) {
  g_err.clear();
  if (!bytes_per_s || !sm_hz) return fail(BSOLVE_ERR_INVALID, "NULL output");
  int prev = -1;
  cudaGetDevice(&prev);
  if (device < 0) device = prev;
  CUDA_TRY(cudaSetDevice(device));
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, device));
  const int grid = prop.multiProcessorCount * 2, iters = 1 << 14;
  constexpr int NT = 512;
  double *sink = nullptr;
  long long *cyc = nullptr;
  CUDA_TRY(cudaMalloc(&sink, sizeof(double) * grid));
  CUDA_TRY(cudaMalloc(&cyc, sizeof(long long) * grid));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  smem_probe_kernel<NT><<<grid, NT>>>(64, sink, cyc);  // warm-up
  cudaEventRecord(e0);
  smem_probe_kernel<NT><<<grid, NT>>>(iters, sink, cyc);
  cudaEventRecord(e1);
  cudaError_t e = cudaEventSynchronize(e1);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  std::vector<long long> hc(grid);
  cudaMemcpy(hc.data(), cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
  cudaFree(sink);
  cudaFree(cyc);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (prev >= 0) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "smem probe: %s", cudaGetErrorString(e));
  const double bytes = (double)grid * NT * iters * 4 * 32;
  *bytes_per_s = bytes / (ms * 1e-3);
  long long mx = 0;
  for (long long c : hc) mx = std::max(mx, c);
  *sm_hz = (double)mx / (ms * 1e-3);
  return BSOLVE_OK;
}

extern "C" int bsolve_probe_fp64(int device, double *flops_per_s, double *sm_hz) {
  g_err.clear();
  if (!flops_per_s || !sm_hz) return fail(BSOLVE_ERR_INVALID, "NULL output");
  int prev = -1;
  cudaGetDevice(&prev);
  if (device < 0) device = prev;
  CUDA_TRY(cudaSetDevice(device));
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, device));
  constexpr int NT = 256;
  const int grid = prop.multiProcessorCount * 4, iters = 1 << 15;
  double *sink = nullptr;
  long long *cyc = nullptr;
  CUDA_TRY(cudaMalloc(&sink, sizeof(double) * grid));
  CUDA_TRY(cudaMalloc(&cyc, sizeof(long long) * grid));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  fp64_probe_kernel<NT><<<grid, NT>>>(256, 1.0, sink, cyc);  // warm-up
  cudaEventRecord(e0);
  fp64_probe_kernel<NT><<<grid, NT>>>(iters, 1.0, sink, cyc);
  cudaEventRecord(e1);
  cudaError_t e = cudaEventSynchronize(e1);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  std::vector<long long> hc(grid);
  cudaMemcpy(hc.data(), cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
  cudaFree(sink);
  cudaFree(cyc);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (prev >= 0) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(BSOLVE_ERR_CUDA, "fp64 probe: %s", cudaGetErrorString(e));
  *flops_per_s = (double)grid * NT * iters * 8 * 2 / (ms * 1e-3);
  long long mx = 0;
  for (long long c : hc) mx = std::max(mx, c);
  *sm_hz = (double)mx / (ms * 1e-3);
  return BSOLVE_OK;
}
