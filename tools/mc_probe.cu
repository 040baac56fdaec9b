// Probe: NVSwitch multicast object with the visible device(s); multimem.st round trip.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#define CK(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char* s; cuGetErrorString(r_, &s); printf("FAIL %s: %s\n", #x, s); return 1; } } while (0)
__global__ void st(double* mc, int n, double base) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) { double v = base + i; asm volatile("multimem.st.relaxed.sys.global.f64 [%0], %1;" :: "l"(mc + i), "d"(v) : "memory"); }
}
int main() {
  CK(cuInit(0));
  int ndev = 0; cuDeviceGetCount(&ndev);
  CUdevice d; CK(cuDeviceGet(&d, 0));
  int mc = -1; cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, d);
  printf("devices %d multicast_supported %d\n", ndev, mc);
  int p2p = 0; if (ndev > 1) cudaDeviceCanAccessPeer(&p2p, 0, 1); printf("p2p01 %d\n", p2p);
  cudaFree(0);
  if (!mc) return 0;
  CUmulticastObjectProp prop; memset(&prop, 0, sizeof prop);
  prop.numDevices = 1; prop.size = 2 << 20; prop.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  if (getenv("MC_FABRIC")) prop.handleTypes = CU_MEM_HANDLE_TYPE_FABRIC;
  size_t gran = 0; CK(cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  printf("gran %zu\n", gran);
  prop.size = ((prop.size + gran - 1) / gran) * gran;
  CUmemGenericAllocationHandle mh; CK(cuMulticastCreate(&mh, &prop));
  CK(cuMulticastAddDevice(mh, d));
  CUmemAllocationProp ap; memset(&ap, 0, sizeof ap);
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED; ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ap.location.id = 0;
  CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, prop.size, &ap, 0));
  CK(cuMulticastBindMem(mh, 0, ph, 0, prop.size, 0));
  CUdeviceptr uc, mcp;
  CK(cuMemAddressReserve(&uc, prop.size, gran, 0, 0)); CK(cuMemMap(uc, prop.size, 0, ph, 0));
  CK(cuMemAddressReserve(&mcp, prop.size, gran, 0, 0)); CK(cuMemMap(mcp, prop.size, 0, mh, 0));
  CUmemAccessDesc ad; ad.location = ap.location; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(uc, prop.size, &ad, 1)); CK(cuMemSetAccess(mcp, prop.size, &ad, 1));
  int n = 1 << 16;
  st<<<n / 256, 256>>>((double*)mcp, n, 3.0);
  cudaError_t e = cudaDeviceSynchronize(); printf("kernel %s\n", cudaGetErrorString(e));
  static double h[1 << 16]; cudaMemcpy(h, (void*)uc, n * 8, cudaMemcpyDeviceToHost);
  int bad = 0; for (int i = 0; i < n; ++i) bad += h[i] != 3.0 + i;
  printf("multimem round trip bad=%d\n", bad);
  return 0;
}
