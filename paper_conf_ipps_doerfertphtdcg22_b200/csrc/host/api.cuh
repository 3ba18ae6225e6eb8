// libomprt host side: lifecycle, status, Fig. 5 host function, kernel introspection.
#pragma once
#include "runtime.cuh"

using namespace omprt_host;

extern "C" int omprt_init(int device, const omprt_options* opt) {
  std::lock_guard<std::mutex> lk(g_mu);
  OMPRT_CHECK_ARG(device >= 0 && device < kMaxDevices, "bad device %d", device);
  Workspace& w = g_ws[device];
  if (w.inited) return OMPRT_OK;
  OMPRT_CUDA_TRY(cudaSetDevice(device));
  omprt_options o{65536, 4096, 1u << 20};
  if (opt) {
    if (opt->pool_bytes_per_team) o.pool_bytes_per_team = opt->pool_bytes_per_team;
    if (opt->pool_teams) o.pool_teams = opt->pool_teams;
    if (opt->max_teams) o.max_teams = opt->max_teams;
  }
  OMPRT_CHECK_ARG(o.pool_bytes_per_team % omprt::kStackAlign == 0 &&
                      o.pool_bytes_per_team <= (1u << 30),
                  "pool_bytes_per_team must be a multiple of 16 below 1 GiB");
  w.opt = o;
  const char* env = getenv("OMPRT_DEBUG");
  w.debug_bits = env ? (unsigned)strtoul(env, nullptr, 0) : 0u;
  if (cudaMalloc(&w.partials, 8 * o.max_teams) != cudaSuccess ||
      cudaMalloc(&w.tickets, 64 * sizeof(unsigned)) != cudaSuccess ||
      cudaMalloc(&w.scratch_u64, 8 * sizeof(uint64_t)) != cudaSuccess ||
      cudaMalloc(&w.pool, o.pool_bytes_per_team * o.pool_teams) != cudaSuccess) {
    cudaGetLastError();
    return set_error(OMPRT_E_NOMEM, "omprt_init: device allocation failed");
  }
  OMPRT_CUDA_TRY(cudaMemset(w.tickets, 0, 64 * sizeof(unsigned)));
  OMPRT_CUDA_TRY(cudaHostAlloc(&w.err_host, 8 * sizeof(int), cudaHostAllocMapped));
  memset(w.err_host, 0, 8 * sizeof(int));
  OMPRT_CUDA_TRY(cudaHostGetDevicePointer(&w.err_dev, w.err_host, 0));
  omprt::DeviceEnv env_dev{w.pool, o.pool_bytes_per_team, o.pool_teams, w.err_dev,
                           w.err_dev + 1, w.debug_bits, 0u};
  OMPRT_CUDA_TRY(cudaMemcpyToSymbol(omprt_env, &env_dev, sizeof env_dev));
  // No L2 set-aside for persisting accesses by default: a reserved set-aside slows every
  // streaming kernel (SU(3) 32^4: 0.24 -> 0.71 ms with the 82.9 MB maximum reserved,
  // profiles/l2_probe_x07.txt).  omprt_l2_set_aside opts in (the XS flat launches' window).
  w.l2_persist_bytes = 0;
  cudaGetLastError();  // a device without the set-aside just runs without windows
  OMPRT_CUDA_TRY(cudaDeviceSynchronize());
  w.inited = true;
  return OMPRT_OK;
}

extern "C" int omprt_fini(int device) {
  std::lock_guard<std::mutex> lk(g_mu);
  OMPRT_CHECK_ARG(device >= 0 && device < kMaxDevices, "bad device %d", device);
  Workspace& w = g_ws[device];
  if (!w.inited) return OMPRT_OK;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(device);
  cudaDeviceSynchronize();
  cudaFree(w.partials);
  cudaFree(w.tickets);
  cudaFree(w.scratch_u64);
  cudaFree(w.pool);
  cudaFree(w.xs_buf[0]);
  cudaFree(w.xs_buf[1]);
  cudaFree(w.xs_built[0]);
  cudaFree(w.xs_built[1]);
  cudaFree(w.dev_ck);
  cudaFree(w.derive_tmp);
  cudaFree(w.e2e_ver);
  if (w.pinned_ck) cudaFreeHost(w.pinned_ck);
  for (int k = 0; k < 2; ++k) {
    if (w.copy_done[k]) cudaEventDestroy(w.copy_done[k]);
    if (w.compute_done[k]) cudaEventDestroy(w.compute_done[k]);
  }
  if (w.copy_stream) cudaStreamDestroy(w.copy_stream);
  cudaFreeHost(w.err_host);
  omprt::DeviceEnv zero{};
  cudaMemcpyToSymbol(omprt_env, &zero, sizeof zero);
  w = Workspace{};
  cudaSetDevice(prev);
  return OMPRT_OK;
}

extern "C" int omprt_l2_set_aside(uint64_t bytes, uint64_t* granted) {
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  int dev = 0, max_persist = 0;
  OMPRT_CUDA_TRY(cudaGetDevice(&dev));
  OMPRT_CUDA_TRY(cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, dev));
  const size_t want = std::min<uint64_t>(bytes, (uint64_t)std::max(max_persist, 0));
  OMPRT_CUDA_TRY(cudaDeviceSynchronize());
  OMPRT_CUDA_TRY(cudaCtxResetPersistingL2Cache());
  OMPRT_CUDA_TRY(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want));
  size_t got = 0;
  OMPRT_CUDA_TRY(cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize));
  w->l2_persist_bytes = got;
  if (granted) *granted = got;
  return OMPRT_OK;
}

extern "C" int omprt_l2_reset_persisting(void) {
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CUDA_TRY(cudaCtxResetPersistingL2Cache());
  return OMPRT_OK;
}

extern "C" int omprt_device_status(int device, int* code, int* info) {
  OMPRT_CHECK_ARG(device >= 0 && device < kMaxDevices && code, "bad arguments");
  Workspace& w = g_ws[device];
  if (!w.inited) return set_error(OMPRT_E_NOTINIT, "device %d not initialized", device);
  *code = ((volatile int*)w.err_host)[0];
  if (info)
    for (int k = 0; k < 4; k++) info[k] = ((volatile int*)w.err_host)[1 + k];
  return OMPRT_OK;
}

extern "C" int omprt_last_error(char* buf, size_t n) {
  size_t len = strlen(g_last_error);
  if (buf && n) {
    size_t m = len < n - 1 ? len : n - 1;
    memcpy(buf, g_last_error, m);
    buf[m] = 0;
  }
  return (int)len;
}

// Fig. 5: IV = BId*NumThreads + TId, stride NumBlocks*NumThreads.
extern "C" int omprt_static_owner(int64_t iv, int64_t n, int32_t teams, int32_t threads,
                                  int32_t* team, int32_t* thread) {
  OMPRT_CHECK_ARG(teams > 0 && threads > 0 && iv >= 0 && iv < n && team && thread,
                  "omprt_static_owner: bad arguments");
  const int64_t g = iv % ((int64_t)teams * threads);
  *team = (int32_t)(g / threads);
  *thread = (int32_t)(g % threads);
  return OMPRT_OK;
}

extern "C" int omprt_kernel_count(void) { return (int)registry().size(); }

extern "C" const char* omprt_kernel_name(int id) {
  if (id < 0 || id >= (int)registry().size()) return nullptr;
  return registry()[id].name;
}

extern "C" int omprt_kernel_attrs(int id, int* regs, int* static_smem, int* local_bytes,
                                  int* max_threads) {
  OMPRT_CHECK_ARG(id >= 0 && id < (int)registry().size(), "bad kernel id %d", id);
  cudaFuncAttributes a{};
  OMPRT_CUDA_TRY(cudaFuncGetAttributes(&a, registry()[id].fn));
  if (regs) *regs = a.numRegs;
  if (static_smem) *static_smem = (int)a.sharedSizeBytes;
  if (local_bytes) *local_bytes = (int)a.localSizeBytes;
  if (max_threads) *max_threads = a.maxThreadsPerBlock;
  return OMPRT_OK;
}

extern "C" int omprt_kernel_occupancy(int id, int threads, int dyn_smem, int* blocks_per_sm) {
  OMPRT_CHECK_ARG(id >= 0 && id < (int)registry().size(), "bad kernel id %d", id);
  OMPRT_CHECK_ARG(threads > 0 && dyn_smem >= 0 && blocks_per_sm, "bad arguments");
  OMPRT_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, registry()[id].fn,
                                                               threads, (size_t)dyn_smem));
  return OMPRT_OK;
}
