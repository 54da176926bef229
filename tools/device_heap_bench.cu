// Device-heap `new` throughput (the CUDA baseline's allocator) vs the
// objects already live: one thread per `new`, 2^lg objects in chunks of 2^chunk.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/dhb tools/device_heap_bench.cu
//   /tmp/dhb <heap GiB> <lg> <chunk lg>     (results: profiles/device_heap_r2.md)
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>
struct B { virtual __device__ void f(){} int v; };
struct D0 : B { __device__ D0(int x){v=x;} __device__ void f() override {v+=1;} };
struct D1 : B { __device__ D1(int x){v=x;} __device__ void f() override {v+=2;} };
__global__ void knew(uint64_t off, uint64_t n, uint64_t* out){
  uint64_t i=off+blockIdx.x*(uint64_t)blockDim.x+threadIdx.x; if(i>=n) return;
  B* o = (i&1)? (B*)new D1((int)i) : (B*)new D0((int)i);
  out[i]=(uint64_t)o;
}
int main(int argc,char**argv){
  size_t heap = (size_t)atoll(argv[1])<<30; int lg=atoi(argv[2]); uint64_t chunk = 1ull<<atoi(argv[3]);
  cudaDeviceSetLimit(cudaLimitMallocHeapSize, heap);
  uint64_t n=1ull<<lg; uint64_t* out; cudaMalloc(&out, 8*n);
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  for(uint64_t off=0; off<n; off+=chunk){
    uint64_t m = n-off<chunk? n-off:chunk;
    cudaEventRecord(a); knew<<<(unsigned)((m+255)/256),256>>>(off, off+m,out); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms,a,b);
    printf("heap %zuG n=2^%d chunk@%llu: %.1f ms (%.2f M/s) %s\n", heap>>30, lg, (unsigned long long)off, ms, m/ms/1e3, cudaGetErrorString(cudaGetLastError())); fflush(stdout);
  }
  uint64_t* h=(uint64_t*)malloc(8*n); cudaMemcpy(h,out,8*n,cudaMemcpyDeviceToHost); uint64_t nul=0; for(uint64_t i=0;i<n;i++) nul+=h[i]==0; printf("nulls %llu\n",(unsigned long long)nul);
}
