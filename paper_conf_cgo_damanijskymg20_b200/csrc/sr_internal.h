// sr_internal.h -- host-side internals shared by the libsr translation units.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>
#include <string>

#include "../../include/sr.h"

namespace sr {

// MCML CTA size (and __launch_bounds__ of its kernels): 2 CTAs x 640 threads at
// <= 48 registers (40 warps / SM) measured best on B200 (tools/exp_occ2.sh:
// 512 -> 35.6 ms, 576 -> 34.8, 640 -> 34.8, 3 x 416 -> 35.0, 704 (spills) -> 35.7)
#ifndef SR_MCML_MAXT
#define SR_MCML_MAXT 640
#endif

// CTA-size launch bounds of the path-tracer and RSBench kernels
#define SR_PT_MAXT 128
#define SR_RS_MAXT 256

constexpr int kCounters = 16;
constexpr int kSchedWords = 8;  // uint32 per warp

// Resolved workspace layout of one (workload, n_threads).
struct Layout {
  size_t off[5];
  size_t bytes[5];
  size_t total;
};
Layout layout_of(const sr_workload& w, uint64_t n_threads);

struct LaunchCtx {
  cudaStream_t stream;
  char* ws;          // workspace base
  Layout lay;
  int sm_count;
  uint32_t block;    // resolved CTA size
};

// Set the calling thread's sr_last_error() text; returns `code`.
int set_error(int code, const std::string& msg);

// A launcher returning an error of its own (not the driver's) explains it
// here; the text is appended to sr_last_error().
void set_launch_note(const std::string& why);

// The launch configuration of the most recent kernel (sr_last_launch).
void record_launch(uint32_t grid, uint32_t block, uint32_t smem_bytes);

// Each returns a cudaError_t from the launch (cudaGetLastError after it).
cudaError_t launch_divloop(const LaunchCtx& c, const sr_workload& w, uint64_t n, uint32_t iters,
                           uint64_t seed, int mode, uint32_t T);
cudaError_t launch_commoncall(const LaunchCtx& c, const sr_workload& w, uint64_t n,
                              uint32_t iters, uint64_t seed, int mode);
cudaError_t launch_mcml(const LaunchCtx& c, const sr_workload& w, uint64_t n, uint32_t iters,
                        uint64_t seed, int mode, uint32_t T);
cudaError_t launch_rsbench(const LaunchCtx& c, const sr_workload& w, uint64_t n, uint32_t iters,
                           uint64_t seed, int mode, uint32_t T);
cudaError_t launch_pathtrace(const LaunchCtx& c, const sr_workload& w, uint64_t n,
                             uint32_t iters, uint64_t seed, int mode, uint32_t T);

cudaError_t launch_math_eval(cudaStream_t st, int sm_count, int fn, const float* x, float* out,
                             uint64_t n);
cudaError_t launch_fresnel_eval(cudaStream_t st, int sm_count, int variant, float p,
                                const float* x, float* out, uint64_t n);
cudaError_t launch_math_eval_p(cudaStream_t st, int sm_count, int fn, float p, const float* x,
                               float* out, uint64_t n);
cudaError_t launch_pt_query(cudaStream_t st, const void* scene, const float* rays, int64_t* hit,
                            float* t, uint64_t n);

// Validation of workload-specific parameters; returns "" when fine.
std::string check_mcml(const sr_mcml_params& p);
std::string check_pathtrace(const sr_pathtrace_params& p, uint64_t n_threads);
size_t pathtrace_perthread_bytes(uint64_t n_threads);
// Remember the header (a PtHeader, 128 bytes) of a scene image written to `dev`.
void register_scene(const void* dev, const void* header);

}  // namespace sr
