// util.cu — small helper kernels (result checksums for the end-to-end path).
#include "vf_internal.h"

namespace vf {
__global__ void k_checksum_i32(const int32_t* __restrict__ v, uint64_t n, long long* out) {
  long long s = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  // 16-byte vector loads over the aligned body
  const uint64_t n4 = n / 4;
  const int4* v4 = reinterpret_cast<const int4*>(v);
  for (uint64_t k = i; k < n4; k += stride) {
    int4 x = v4[k];
    s += (long long)x.x + x.y + x.z + x.w;
  }
  for (uint64_t k = n4 * 4 + i; k < n; k += stride) s += v[k];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(reinterpret_cast<unsigned long long*>(out), (unsigned long long)s);
}
}  // namespace vf

extern "C" vf_status vf_checksum_i32(const int32_t* vals_dev, uint64_t n, long long* out_dev,
                                     void* stream) {
  if (!out_dev || (n && !vals_dev)) return VF_ERR_INVALID;
  if (reinterpret_cast<uintptr_t>(vals_dev) % 16) return VF_ERR_INVALID;
  if (!n) return VF_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint64_t g = (n / 4 + 255) / 256;
  if (g > (uint64_t)sms * 8) g = (uint64_t)sms * 8;
  if (g == 0) g = 1;
  vf::k_checksum_i32<<<(unsigned)g, 256, 0, (cudaStream_t)stream>>>(vals_dev, n, out_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
