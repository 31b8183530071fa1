// debug_kernels.cu — device-side primitives exposed for the parity tests:
// the library's Philox stream and, as an independent cross-check,
// curand_Philox4x32_10 from the CUDA toolkit on the same counters.
#include <cuda_runtime.h>
#include <curand_philox4x32_x.h>

#include "kernels.h"
#include "philox.cuh"

namespace fastpso {
namespace {

__global__ void k_philox_words(PhiloxKey key, unsigned tag, unsigned t, unsigned i, unsigned j0,
                               long long m, unsigned* out, int use_curand) {
  for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < m;
       k += (long long)gridDim.x * blockDim.x) {
    const unsigned j = j0 + (unsigned)k;
    const uint4 ctr = make_uint4(j >> 2, i, t, tag);
    uint4 w;
    if (use_curand) {
      w = curand_Philox4x32_10(ctr, make_uint2(key.k0, key.k1));
    } else {
      w = philox4x32_10(ctr, key);
    }
    const unsigned e = j & 3u;
    out[k] = e == 0 ? w.x : (e == 1 ? w.y : (e == 2 ? w.z : w.w));
  }
}

}  // namespace

cudaError_t debug_philox(unsigned long long seed, unsigned tag, unsigned t, unsigned i,
                         unsigned j0, long long m, unsigned* out_dev, int use_curand,
                         cudaStream_t s) {
  if (m <= 0) return cudaSuccess;
  long long blocks = (m + 255) / 256;
  if (blocks > 4096) blocks = 4096;
  const PhiloxKey key{(unsigned)seed, (unsigned)(seed >> 32)};
  k_philox_words<<<(unsigned)blocks, 256, 0, s>>>(key, tag, t, i, j0, m, out_dev, use_curand);
  return cudaGetLastError();
}

}  // namespace fastpso
