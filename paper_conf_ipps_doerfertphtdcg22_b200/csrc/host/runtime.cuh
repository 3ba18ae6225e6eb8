// libomprt host side: per-device workspace, error reporting, launch helpers.
// Part of the single translation unit src/libomprt.cu (one __constant__ omprt_env).
#pragma once
#include <cuda_runtime.h>

#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "../../../include/omprt.h"
#include "../omprt/device/omprt.cuh"

namespace omprt_host {

thread_local char g_last_error[512] = "";

inline int set_error(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_last_error, sizeof g_last_error, fmt, ap);
  va_end(ap);
  return code;
}

#define OMPRT_CUDA_TRY(expr)                                                            \
  do {                                                                                  \
    cudaError_t _e = (expr);                                                            \
    if (_e != cudaSuccess)                                                              \
      return ::omprt_host::set_error(OMPRT_E_CUDA, "%s failed: %s (%s:%d)", #expr,        \
                                     cudaGetErrorString(_e), __FILE__, __LINE__);       \
  } while (0)

#define OMPRT_CHECK_ARG(cond, ...)                                                      \
  do {                                                                                  \
    if (!(cond)) return ::omprt_host::set_error(OMPRT_E_INVAL, __VA_ARGS__);           \
  } while (0)

// Library-owned per-device state (ownership rule of include/omprt.h).
struct Workspace {
  bool inited = false;
  void* partials = nullptr;       // league-reduction partials, 8 B x max_teams
  unsigned* tickets = nullptr;    // league-reduction tickets (zeroed)
  unsigned char* pool = nullptr;  // smem-stack fallback pool
  int* err_host = nullptr;        // mapped pinned: error word + 4 info ints
  int* err_dev = nullptr;
  uint64_t* scratch_u64 = nullptr;  // 8 slots of device scratch (e2e checksum, ...)
  omprt_options opt{};
  unsigned debug_bits = 0;
  // e2e (omprt_xs_run_host*) device copies of the tables, two slots (double buffering
  // across steps), grown on demand; a copy stream, per-slot events, pinned checksums
  void* xs_buf[2] = {nullptr, nullptr};
  size_t xs_buf_bytes = 0;
  // ... and one buffer for the tables built on the device (written and read on the compute
  // stream only, so one copy serves every step, and the L2 window stays on one range)
  void* xs_built[2] = {nullptr, nullptr};  // device-built layouts, one set per table slot
  size_t xs_built_bytes = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t copy_done[2] = {nullptr, nullptr};
  cudaEvent_t compute_done[2] = {nullptr, nullptr};
  uint64_t* pinned_ck = nullptr;     // [kMaxE2ESteps]
  uint64_t* dev_ck = nullptr;        // [kMaxE2ESteps]
  // omprt_xs_run_host_steps with derived tables: omprt_xs_derive scratch (grown on demand)
  void* derive_tmp = nullptr;
  size_t derive_tmp_bytes = 0;
  // flattened e2e steps: per-lookup verification scratch, summed by K11 (u64 entries)
  uint64_t* e2e_ver = nullptr;
  size_t e2e_ver_n = 0;
  // L2 set-aside for persisting accesses (cudaLimitPersistingL2CacheSize), granted by omprt_l2_set_aside
  size_t l2_persist_bytes = 0;
};
constexpr int kMaxE2ESteps = 1024;

constexpr int kMaxDevices = 64;
Workspace g_ws[kMaxDevices];
std::mutex g_mu;

inline int current_ws(Workspace** out) {
  int dev = 0;
  OMPRT_CUDA_TRY(cudaGetDevice(&dev));
  if (dev < 0 || dev >= kMaxDevices || !g_ws[dev].inited)
    return set_error(OMPRT_E_NOTINIT, "omprt_init was not called for device %d", dev);
  *out = &g_ws[dev];
  return OMPRT_OK;
}

inline cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

inline int check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess)
    return set_error(OMPRT_E_CUDA, "launch of %s failed: %s", what, cudaGetErrorString(e));
  return OMPRT_OK;
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ---- kernel registry (omprt_kernel_attrs) ---------------------------------------------
struct KernelEntry {
  const char* name;
  const void* fn;
};
inline std::vector<KernelEntry>& registry() {
  static std::vector<KernelEntry> r;
  return r;
}
struct Register {
  Register(const char* name, const void* fn) { registry().push_back({name, fn}); }
};
#define OMPRT_REGISTER_KERNEL(NAME, ...) \
  static ::omprt_host::Register _omprt_reg_##NAME(#NAME, (const void*)(__VA_ARGS__));

}  // namespace omprt_host
