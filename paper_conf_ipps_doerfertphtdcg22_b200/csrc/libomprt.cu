// libomprt.so: the whole library is one translation unit, so the header-only device
// runtime is compiled (and optimized) together with every kernel that uses it, and
// the per-device environment has a single __constant__ definition.
#include "host/runtime.cuh"
#include "host/api.cuh"
#include "kernels/axpy.cuh"
#include "kernels/axpy_chunk.cuh"
#include "kernels/generic.cuh"
#include "kernels/xsbench.cuh"
#include "kernels/xs_derive.cuh"
#include "kernels/rs_su3.cuh"
#include "kernels/su3_staged.cuh"
#include "kernels/lockstep_probe.cuh"
#include "kernels/peaks.cuh"
