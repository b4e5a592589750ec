// sr_api.cu -- the C ABI of include/sr.h: validation, context, workspace
// layout, dispatch to the kernel families, error mapping.  No exception and
// no CUDA error crosses the ABI; every failure becomes a negative sr_status
// plus a thread-local message.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>

#include "sr_internal.h"

namespace sr {
namespace {

thread_local std::string g_err;

struct Context {
  bool live = false;
  int device = -1;
  cudaStream_t stream = nullptr;
  char* ws = nullptr;
  size_t ws_bytes = 0;
  int sm_count = 0;
  // last run, for sr_tally
  bool have_run = false;
  Layout last{};
};
Context g_ctx;
std::mutex g_mu;
uint32_t g_launch[4];  // grid, block, smem, kernels of the current/last sr_run

int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}
thread_local std::string g_note;  // launcher's explanation of its own error return
int fail_cuda(cudaError_t e, const char* where) {
  cudaGetLastError();  // clear sticky-free errors
  std::string msg = std::string(where) + ": " + cudaGetErrorName(e) + ": " + cudaGetErrorString(e);
  if (!g_note.empty()) msg += " (" + g_note + ")";
  g_note.clear();
  return fail(SR_E_CUDA, msg);
}
size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

// __launch_bounds__ of each workload's kernels
uint32_t max_block(int kind) {
  switch (kind) {
    case SR_WL_MCML: return SR_MCML_MAXT;
    case SR_WL_PATHTRACE: return SR_PT_MAXT;
    case SR_WL_RSBENCH: return SR_RS_MAXT;
    default: return 1024;
  }
}

std::string check_workload(const sr_workload* w, uint64_t n_threads) {
  if (!w) return "workload is NULL";
  if (n_threads == 0) return "n_threads must be >= 1";
  if (w->block_threads != 0 &&
      (w->block_threads % 32 != 0 || w->block_threads < 32 || w->block_threads > 1024))
    return "block_threads must be 0 or a multiple of 32 in [32, 1024]";
  if (w->block_threads > max_block(w->kind))
    return "block_threads exceeds this workload's kernels' launch bound (" +
           std::to_string(max_block(w->kind)) + ")";
  if (w->flags & ~(SR_F_SCHED | SR_F_STATIC | SR_F_COARSE | SR_F_NOSPLIT | SR_F_MATGROUP |
                   SR_F_POOL))
    return "unknown flags";
  switch (w->kind) {
    case SR_WL_DIVLOOP:
      if (w->divloop.fma_count % 8 != 0) return "divloop.fma_count must be a multiple of 8";
      if (w->divloop.prolog_batch > 1 && w->divloop.prolog_batch != 64)
        return "divloop.prolog_batch must be 0, 1 or 64";
      if ((w->flags & SR_F_POOL) && w->divloop.prolog_batch != 64)
        return "divloop: SR_F_POOL needs prolog_batch = 64";
      if (w->divloop.pool_split > 1 &&
          (w->divloop.pool_split != 2 && w->divloop.pool_split != 4))
        return "divloop.pool_split must be 0, 1, 2 or 4";
      if (w->divloop.prolog_batch == 64 && w->block_threads > 512)
        return "divloop.prolog_batch = 64 needs block_threads <= 512 (64 shared-memory floats "
               "per thread)";
      if (n_threads > (1ull << 40)) return "n_threads too large";
      return "";
    case SR_WL_COMMONCALL:
      if (w->commoncall.fma_count % 8 != 0) return "commoncall.fma_count must be a multiple of 8";
      if (n_threads > (1ull << 40)) return "n_threads too large";
      return "";
    case SR_WL_MCML:
      return check_mcml(w->mcml);
    case SR_WL_PATHTRACE:
      if (w->flags & SR_F_POOL) {
        if (w->flags & (SR_F_COARSE | SR_F_NOSPLIT | SR_F_MATGROUP))
          return "pathtrace: SR_F_POOL is for the split merge (not with SR_F_COARSE, "
                 "SR_F_NOSPLIT or SR_F_MATGROUP)";
        if (w->pathtrace.pool_spp == 0 || w->pathtrace.pool_spp > 4096)
          return "pathtrace: SR_F_POOL needs pool_spp in [1, 4096]";
      }
      return check_pathtrace(w->pathtrace, n_threads);
    case SR_WL_RSBENCH:
      if (w->rsbench.fma_count % 8 != 0) return "rsbench.fma_count must be a multiple of 8";
      if (w->rsbench.prolog_fma % 8 != 0 || w->rsbench.prolog_fma > 65536)
        return "rsbench.prolog_fma must be a multiple of 8 in [0, 65536]";
      if (n_threads > (1ull << 40)) return "n_threads too large";
      return "";
    default:
      return "unknown workload kind " + std::to_string(w->kind);
  }
}

uint32_t default_block(const sr_workload& w) {
  if (w.block_threads) return w.block_threads;
  switch (w.kind) {
    case SR_WL_DIVLOOP: return 64;
    case SR_WL_COMMONCALL: return 256;
    case SR_WL_MCML: return SR_MCML_MAXT;
    case SR_WL_RSBENCH: return 256;
    default: return 128;
  }
}

}  // namespace

int set_error(int code, const std::string& msg) { return fail(code, msg); }

void record_launch(uint32_t grid, uint32_t block, uint32_t smem_bytes) {
  g_launch[0] = grid;
  g_launch[1] = block;
  g_launch[2] = smem_bytes;
  g_launch[3] += 1;
}

Layout layout_of(const sr_workload& w, uint64_t n) {
  Layout L{};
  size_t per = 0, grid = 0;
  switch (w.kind) {
    case SR_WL_DIVLOOP: per = 8 * n; break;
    case SR_WL_RSBENCH: per = 8 * n; break;
    case SR_WL_COMMONCALL: per = 4 * n; break;
    case SR_WL_MCML: grid = 8ull * ((uint64_t)w.mcml.nz * w.mcml.nr + 2ull * w.mcml.nr); break;
    case SR_WL_PATHTRACE: per = pathtrace_perthread_bytes(n); break;
    default: break;
  }
  const uint32_t block = default_block(w);
  // schedule counters: one record per launched warp of the largest grid any kernel
  // uses (a partial last CTA launches whole warps past n; kernels also skip the
  // record of a warp whose first thread is >= n)
  uint64_t warps = ((n + block - 1) / block) * (block / 32);
  if (w.kind == SR_WL_MCML || w.kind == SR_WL_PATHTRACE) {
    const uint64_t gw = ((n + block - 1) / block) * (block / 32);
    const uint64_t dyn = (uint64_t)2048 * 1024 / 32;  // >= any persistent grid (148 SMs x 2048)
    warps = gw > dyn ? gw : dyn;
  }
  const size_t sched = (w.flags & SR_F_SCHED) ? 4ull * kSchedWords * warps : 0;
  // SCRATCH: 256 bytes of claim counters, then (PATHTRACE + SR_F_POOL) the per-path
  // radiance of up to pool_spp samples per pixel, 3 floats each
  const size_t pool_buf = (w.kind == SR_WL_PATHTRACE && (w.flags & SR_F_POOL))
                              ? 12ull * n * w.pathtrace.pool_spp : 0;
  const size_t bytes[5] = {per, grid, 8ull * kCounters, sched, 256 + pool_buf};
  size_t off = 0;
  for (int i = 0; i < 5; ++i) {
    // GRID and COUNTERS adjacent (GRID is a multiple of 8 bytes; no padding
    // between them so one int64 all-reduce covers both)
    if (i == SR_T_COUNTERS && bytes[SR_T_GRID] > 0) {
      L.off[i] = L.off[SR_T_GRID] + bytes[SR_T_GRID];
      L.bytes[i] = bytes[i];
      off = align256(L.off[i] + bytes[i]);
      continue;
    }
    L.off[i] = off;
    L.bytes[i] = bytes[i];
    off = align256(off + bytes[i]);
  }
  L.total = off;
  return L;
}

void set_launch_note(const std::string& why) { g_note = why; }

}  // namespace sr

using namespace sr;

extern "C" {

const char* sr_last_error(void) { return g_err.c_str(); }

const char* sr_build_info(void) {
#ifndef SR_NVCC_VERSION
#define SR_NVCC_VERSION "unknown"
#endif
  return "libsr sm_100a nvcc " SR_NVCC_VERSION " --fmad=false -O3 -lineinfo";
}

int sr_math_eval(int fn, const float* x_dev, float* out_dev, uint64_t n) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  if (fn < SR_FN_LOGF || fn > SR_FN_EXPENSIVE_2000) return fail(SR_E_INVALID, "unknown fn");
  if (n && (!x_dev || !out_dev)) return fail(SR_E_INVALID, "NULL array");
  if (!g_ctx.live) return fail(SR_E_STATE, "sr_math_eval before sr_init");
  if (!n) return SR_OK;
  const cudaError_t e = launch_math_eval(g_ctx.stream, g_ctx.sm_count, fn, x_dev, out_dev, n);
  if (e != cudaSuccess) return fail_cuda(e, "sr_math_eval");
  return SR_OK;
}

int sr_math_eval_p(int fn, float p, const float* x_dev, float* out_dev, uint64_t n) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  const bool fres = fn >= SR_FNP_FRESNEL && fn < SR_FNP_FRESNEL + 8;
  if (!fres && (fn < SR_FNP_DIV_XP || fn > SR_FNP_DIV2_XP)) return fail(SR_E_INVALID, "unknown fn");
  if (n && (!x_dev || !out_dev)) return fail(SR_E_INVALID, "NULL array");
  if (!g_ctx.live) return fail(SR_E_STATE, "sr_math_eval_p before sr_init");
  if (!n) return SR_OK;
  const cudaError_t e =
      fres ? launch_fresnel_eval(g_ctx.stream, g_ctx.sm_count, fn - SR_FNP_FRESNEL, p, x_dev,
                                 out_dev, n)
           : launch_math_eval_p(g_ctx.stream, g_ctx.sm_count, fn, p, x_dev, out_dev, n);
  if (e != cudaSuccess) return fail_cuda(e, "sr_math_eval_p");
  return SR_OK;
}

int sr_pt_closest(const void* scene_dev, const float* rays_dev, int64_t* hit_dev, float* t_dev,
                  uint64_t n) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  if (!scene_dev || (n && (!rays_dev || !hit_dev || !t_dev)))
    return fail(SR_E_INVALID, "NULL array");
  if (!g_ctx.live) return fail(SR_E_STATE, "sr_pt_closest before sr_init");
  const cudaError_t e = launch_pt_query(g_ctx.stream, scene_dev, rays_dev, hit_dev, t_dev, n);
  if (e == cudaErrorInvalidValue) return fail(SR_E_INVALID, "scene_dev is not a scene image");
  if (e != cudaSuccess) return fail_cuda(e, "sr_pt_closest");
  return SR_OK;
}

int sr_last_launch(uint32_t out[4]) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  if (!out) return fail(SR_E_INVALID, "out is NULL");
  if (!g_ctx.have_run) return fail(SR_E_STATE, "no sr_run since sr_init");
  for (int i = 0; i < 4; ++i) out[i] = g_launch[i];
  return SR_OK;
}

int sr_init(int device, void* cuda_stream, void* workspace_dev, size_t workspace_bytes) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  if (device < 0) return fail(SR_E_INVALID, "device must be >= 0");
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess) return fail_cuda(e, "sr_init: cudaGetDeviceCount");
  if (device >= n) return fail(SR_E_INVALID, "device out of range");
  if ((e = cudaSetDevice(device)) != cudaSuccess) return fail_cuda(e, "sr_init: cudaSetDevice");
  int sms = 0;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device)) != cudaSuccess)
    return fail_cuda(e, "sr_init: cudaDeviceGetAttribute");
  if (workspace_bytes && !workspace_dev)
    return fail(SR_E_INVALID, "workspace_dev is NULL but workspace_bytes > 0");
  g_ctx.live = true;
  g_ctx.device = device;
  g_ctx.stream = static_cast<cudaStream_t>(cuda_stream);
  g_ctx.ws = static_cast<char*>(workspace_dev);
  g_ctx.ws_bytes = workspace_bytes;
  g_ctx.sm_count = sms;
  g_ctx.have_run = false;
  return SR_OK;
}

size_t sr_workspace_bytes(const sr_workload* w, uint64_t n_threads) {
  if (!check_workload(w, n_threads).empty()) return 0;
  return layout_of(*w, n_threads).total;
}

int sr_workspace_region(const sr_workload* w, uint64_t n_threads, int what, size_t* offset,
                        size_t* bytes) {
  g_err.clear();
  const std::string why = check_workload(w, n_threads);
  if (!why.empty()) return fail(SR_E_INVALID, why);
  if (what < 0 || what > SR_T_SCRATCH) return fail(SR_E_INVALID, "unknown region");
  const Layout L = layout_of(*w, n_threads);
  if (offset) *offset = L.off[what];
  if (bytes) *bytes = L.bytes[what];
  return SR_OK;
}

int sr_run(const sr_workload* w, uint64_t n_threads, uint32_t iters, uint64_t seed, int mode,
           uint32_t threshold) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  // arguments first (so validation is testable without a device), then state
  const std::string why = check_workload(w, n_threads);
  if (!why.empty()) return fail(SR_E_INVALID, why);
  if (mode != SR_PDOM && mode != SR_SPEC_LOOP && mode != SR_SPEC_CALL)
    return fail(SR_E_INVALID, "unknown mode");
  if (mode == SR_SPEC_CALL && w->kind != SR_WL_COMMONCALL)
    return fail(SR_E_INVALID, "SR_SPEC_CALL is only valid for SR_WL_COMMONCALL");
  if (mode == SR_SPEC_LOOP && w->kind == SR_WL_COMMONCALL)
    return fail(SR_E_INVALID, "SR_SPEC_LOOP is not valid for SR_WL_COMMONCALL");
  if (threshold > 32) return fail(SR_E_INVALID, "threshold must be in [0, 32]");
  if (w->kind == SR_WL_PATHTRACE && (w->flags & SR_F_POOL) && iters > w->pathtrace.pool_spp)
    return fail(SR_E_INVALID, "pathtrace: iters (spp) exceeds pathtrace.pool_spp, the samples "
                              "per pixel the workspace holds with SR_F_POOL");
  if (mode == SR_SPEC_CALL && threshold != 0 && threshold != 32)
    return fail(SR_E_INVALID, "SR_SPEC_CALL waits for all lanes: threshold must be 0 or 32");
  const uint32_t T = threshold == 0 ? 32u : threshold;
  if (iters != 0 && n_threads > (1ull << 63) / iters)
    return fail(SR_E_INVALID, "n_threads * iters overflows");
  if (w->task_offset > ~0ull - n_threads * (uint64_t)(iters ? iters : 1))
    return fail(SR_E_INVALID, "task_offset + tasks overflows 2^64");
  if (!g_ctx.live) return fail(SR_E_STATE, "sr_run before sr_init (or after sr_finalize)");
  const Layout L = layout_of(*w, n_threads);
  if (L.total > g_ctx.ws_bytes)
    return fail(SR_E_NOMEM, "workspace has " + std::to_string(g_ctx.ws_bytes) + " bytes, run needs " +
                                std::to_string(L.total));
  LaunchCtx c{g_ctx.stream, g_ctx.ws, L, g_ctx.sm_count, default_block(*w)};
  cudaError_t e;
  g_launch[3] = 0;
  // zero the outputs of this run (per-thread outputs and the path tracer's per-path
  // radiance are fully overwritten): GRID, COUNTERS, SCHED and SCRATCH's counters lie
  // back to back (layout_of), so one memset node covers them and their alignment
  // padding -- one operation per run instead of up to four keeps the launch overhead
  // of microsecond-scale runs down
  {
    const size_t z0 = L.off[SR_T_GRID];
    const size_t z1 = L.off[SR_T_SCRATCH] + 256;
    if ((e = cudaMemsetAsync(g_ctx.ws + z0, 0, z1 - z0, g_ctx.stream)) != cudaSuccess)
      return fail_cuda(e, "sr_run: cudaMemsetAsync");
  }
  switch (w->kind) {
    case SR_WL_DIVLOOP: e = launch_divloop(c, *w, n_threads, iters, seed, mode, T); break;
    case SR_WL_COMMONCALL: e = launch_commoncall(c, *w, n_threads, iters, seed, mode); break;
    case SR_WL_MCML: e = launch_mcml(c, *w, n_threads, iters, seed, mode, T); break;
    case SR_WL_RSBENCH: e = launch_rsbench(c, *w, n_threads, iters, seed, mode, T); break;
    default: e = launch_pathtrace(c, *w, n_threads, iters, seed, mode, T); break;
  }
  if (e != cudaSuccess) return fail_cuda(e, "sr_run: kernel launch");
  g_ctx.have_run = true;
  g_ctx.last = L;
  return SR_OK;
}

int sr_tally(int what, void* dst, size_t dst_bytes, size_t* written) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  if (written) *written = 0;
  if (!g_ctx.live) return fail(SR_E_STATE, "sr_tally before sr_init (or after sr_finalize)");
  if (!g_ctx.have_run) return fail(SR_E_STATE, "sr_tally before any sr_run");
  if (what < 0 || what > SR_T_SCHED) return fail(SR_E_INVALID, "unknown region");
  const size_t n = g_ctx.last.bytes[what];
  if (n > dst_bytes) return fail(SR_E_NOMEM, "destination smaller than the region");
  if (n && !dst) return fail(SR_E_INVALID, "dst is NULL");
  cudaError_t e;
  if (n && (e = cudaMemcpyAsync(dst, g_ctx.ws + g_ctx.last.off[what], n, cudaMemcpyDefault,
                                g_ctx.stream)) != cudaSuccess)
    return fail_cuda(e, "sr_tally: cudaMemcpyAsync");
  if ((e = cudaStreamSynchronize(g_ctx.stream)) != cudaSuccess)
    return fail_cuda(e, "sr_tally: cudaStreamSynchronize");
  if (written) *written = n;
  return SR_OK;
}

int sr_finalize(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_err.clear();
  g_ctx = Context{};
  return SR_OK;
}

}  // extern "C"
