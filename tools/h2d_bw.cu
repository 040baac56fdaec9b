// PCIe bandwidth of the e2e path's tile copies (HOST_COLMAJOR, pinned): the lower
// nb x nb tiles of an n x n column-major host matrix copied with cudaMemcpy2DAsync
// (nb rows of nb doubles, source pitch n) on 1, 2 or 4 streams, against contiguous
// 8 MiB copies of the same volume.  usage: h2d_bw [n] [nb]
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

// occupies every SM (4 CTAs x 256 threads each, FP64 FMA chains) for ~ms milliseconds
__global__ void busy(double* out, long long cycles) {
  const long long t0 = clock64();
  double x = threadIdx.x;
  while (clock64() - t0 < cycles)
    for (int i = 0; i < 64; ++i) x = fma(x, 0.9999, 1e-7);
  if (x == 12345.0) out[0] = x;
}

int main(int argc, char** argv) {
  const long n = argc > 1 ? atol(argv[1]) : 32768, nb = argc > 2 ? atol(argv[2]) : 1024, T = n / nb;
  const long ntiles = T * (T + 1) / 2, tb = nb * nb * 8;
  double* h = nullptr;
  if (cudaHostAlloc(&h, (size_t)n * n * 8, cudaHostAllocDefault) != cudaSuccess) { printf("pin failed\n"); return 1; }
  for (long i = 0; i < n * n; i += 512) h[i] = 1.0;
  double* d = nullptr;
  cudaMalloc(&d, (size_t)ntiles * tb);
  cudaStream_t st[4];
  for (auto& s : st) cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char* what, int ns, int mode, bool h2d) {
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
      cudaDeviceSynchronize();
      cudaEventRecord(e0, st[0]);
      for (int s = 1; s < ns; ++s) cudaStreamWaitEvent(st[s], e0, 0);
      long t = 0;
      for (long j = 0; j < T; ++j)
        for (long i = j; i < T; ++i, ++t) {
          cudaStream_t s = st[t % ns];
          double* dt = d + t * nb * nb;
          double* ht = h + i * nb + j * nb * n;
          if (mode == 0) {
            if (h2d) cudaMemcpy2DAsync(dt, nb * 8, ht, n * 8, nb * 8, nb, cudaMemcpyHostToDevice, s);
            else cudaMemcpy2DAsync(ht, n * 8, dt, nb * 8, nb * 8, nb, cudaMemcpyDeviceToHost, s);
          } else {
            double* hc = h + t * nb * nb;
            if (h2d) cudaMemcpyAsync(dt, hc, tb, cudaMemcpyHostToDevice, s);
            else cudaMemcpyAsync(hc, dt, tb, cudaMemcpyDeviceToHost, s);
          }
        }
      for (int s = 1; s < ns; ++s) {
        cudaEvent_t ev;
        cudaEventCreate(&ev);
        cudaEventRecord(ev, st[s]);
        cudaStreamWaitEvent(st[0], ev, 0);
      }
      cudaEventRecord(e1, st[0]);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    printf("%-4s %-10s streams=%d: %8.2f ms  %6.1f GB/s\n", h2d ? "H2D" : "D2H", what, ns, best,
           ntiles * tb / (best * 1e-3) / 1e9);
  };
  for (int h2d = 1; h2d >= 0; --h2d)
    for (int ns : {1, 2, 4}) {
      run("2D tiles", ns, 0, h2d);
      run("contig", ns, 1, h2d);
    }
  // copies while every SM is busy (the e2e situation): does the copy need SMs?
  {
    cudaStream_t sb;
    cudaStreamCreateWithFlags(&sb, cudaStreamNonBlocking);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int h2d = 1; h2d >= 0; --h2d) {
      cudaDeviceSynchronize();
      busy<<<sms * 4, 256, 0, sb>>>(reinterpret_cast<double*>(d), 2000000000LL / 10 * 3);  // ~300 ms
      cudaEventRecord(e0, st[0]);
      long t = 0;
      for (long j = 0; j < T; ++j)
        for (long i = j; i < T; ++i, ++t) {
          double* dt = d + t * nb * nb;
          double* ht = h + i * nb + j * nb * n;
          if (h2d) cudaMemcpy2DAsync(dt, nb * 8, ht, n * 8, nb * 8, nb, cudaMemcpyHostToDevice, st[0]);
          else cudaMemcpy2DAsync(ht, n * 8, dt, nb * 8, nb * 8, nb, cudaMemcpyDeviceToHost, st[0]);
        }
      cudaEventRecord(e1, st[0]);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      printf("%s 2D tiles while all SMs busy: %8.2f ms  %6.1f GB/s\n", h2d ? "H2D" : "D2H", ms,
             ntiles * tb / (ms * 1e-3) / 1e9);
      cudaDeviceSynchronize();
    }
  }
  // both directions at once (the e2e overlap): H2D tiles on st[0], D2H tiles on st[1]
  cudaDeviceSynchronize();
  auto t0 = std::chrono::steady_clock::now();
  long t = 0;
  for (long j = 0; j < T; ++j)
    for (long i = j; i < T; ++i, ++t) {
      double* dt = d + t * nb * nb;
      double* ht = h + i * nb + j * nb * n;
      cudaMemcpy2DAsync(dt, nb * 8, ht, n * 8, nb * 8, nb, cudaMemcpyHostToDevice, st[0]);
      double* dt2 = d + ((t + ntiles / 2) % ntiles) * nb * nb;
      cudaMemcpy2DAsync(ht, n * 8, dt2, nb * 8, nb * 8, nb, cudaMemcpyDeviceToHost, st[1]);
    }
  cudaDeviceSynchronize();
  const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  printf("H2D+D2H concurrent 2D tiles: %8.2f ms (%.1f GB/s each way)\n", ms, ntiles * tb / (ms * 1e-3) / 1e9);
  return 0;
}
