// probe_mc.cu -- can this box create an NVLS multicast object (1 device) and run multimem.red?
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#define CK(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char* s; cuGetErrorString(r, &s); printf("%s -> %d %s\n", #x, (int)r, s); return 1; } } while (0)
__global__ void k_red(float* mc, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) asm volatile("multimem.red.relaxed.sys.global.add.f32 [%0], %1;" :: "l"(mc + i), "f"(1.5f) : "memory");
}
int main() {
  CK(cuInit(0));
  CUdevice dev; CK(cuDeviceGet(&dev, 0));
  CUcontext ctx; CK(cuDevicePrimaryCtxRetain(&ctx, dev)); CK(cuCtxSetCurrent(ctx));
  int mc = -1; CK(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
  printf("MULTICAST_SUPPORTED = %d\n", mc);
  CUmulticastObjectProp prop = {};
  prop.numDevices = 1; prop.size = 2 << 20; prop.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  size_t gran = 0; CK(cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  prop.size = ((prop.size + gran - 1) / gran) * gran;
  CUmemGenericAllocationHandle mch; CK(cuMulticastCreate(&mch, &prop));
  CK(cuMulticastAddDevice(mch, dev));
  CUmemAllocationProp ap = {}; ap.type = CU_MEM_ALLOCATION_TYPE_PINNED; ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ap.location.id = 0;
  CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, prop.size, &ap, 0));
  CK(cuMulticastBindMem(mch, 0, ph, 0, prop.size, 0));
  CUdeviceptr uc, mcp;
  CK(cuMemAddressReserve(&uc, prop.size, 0, 0, 0)); CK(cuMemMap(uc, prop.size, 0, ph, 0));
  CK(cuMemAddressReserve(&mcp, prop.size, 0, 0, 0)); CK(cuMemMap(mcp, prop.size, 0, mch, 0));
  CUmemAccessDesc ad = {}; ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad.location.id = 0; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(uc, prop.size, &ad, 1)); CK(cuMemSetAccess(mcp, prop.size, &ad, 1));
  cudaMemset((void*)uc, 0, 1024 * 4);
  k_red<<<4, 256>>>((float*)mcp, 1024); k_red<<<4, 256>>>((float*)mcp, 1024);
  cudaError_t e = cudaDeviceSynchronize(); printf("kernel: %s\n", cudaGetErrorString(e));
  float h[4]; cudaMemcpy(h, (void*)uc, 16, cudaMemcpyDeviceToHost);
  printf("values %g %g %g %g (expect 3)\n", h[0], h[1], h[2], h[3]);
  return 0;
}
