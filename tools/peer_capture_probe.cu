// Probe: can cudaMemcpyPeerAsync / cudaMemcpyAsync(Default) be stream-captured (same device)?
#include <cuda_runtime.h>
#include <cstdio>
int main() {
  double *a, *b;
  cudaMalloc(&a, 1 << 20);
  cudaMalloc(&b, 1 << 20);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  for (int variant = 0; variant < 2; ++variant) {
    cudaGraph_t g = nullptr;
    cudaError_t e0 = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
    cudaError_t e1 = variant == 0 ? cudaMemcpyPeerAsync(b, 0, a, 0, 1 << 20, s)
                                  : cudaMemcpyAsync(b, a, 1 << 20, cudaMemcpyDefault, s);
    cudaError_t e2 = cudaStreamEndCapture(s, &g);
    printf("%s: begin=%s copy=%s end=%s graph=%p\n", variant == 0 ? "cudaMemcpyPeerAsync" : "cudaMemcpyAsync(Default)",
           cudaGetErrorString(e0), cudaGetErrorString(e1), cudaGetErrorString(e2), (void*)g);
    cudaGetLastError();
  }
  return 0;
}
