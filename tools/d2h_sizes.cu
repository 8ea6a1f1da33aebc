// d2h_sizes.cu -- D2H copy-engine rate vs copy size and concurrency (diagnostic tool).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o d2h_sizes d2h_sizes.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                                     \
    do {                                                                                          \
        cudaError_t e = (x);                                                                      \
        if (e != cudaSuccess) {                                                                   \
            fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e));    \
            exit(1);                                                                              \
        }                                                                                         \
    } while (0)

int main() {
    const size_t N = size_t(3) << 30;
    char *d, *h;
    CK(cudaMalloc(&d, N));
    CK(cudaMemset(d, 1, N));
    CK(cudaHostAlloc(&h, N, 0));
    cudaDeviceProp p;
    CK(cudaGetDeviceProperties(&p, 0));
    cudaStream_t s[4];
    for (auto &x : s) CK(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
    cudaEvent_t a, b, j[4];
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    for (auto &x : j) CK(cudaEventCreate(&x));
    printf("{\n \"asyncEngineCount\": %d,\n", p.asyncEngineCount);
    // total bytes fixed at N; pieces of `sz` bytes spread over `ns` streams round-robin
    for (size_t sz : {size_t(16) << 20, size_t(64) << 20, size_t(256) << 20, size_t(512) << 20, size_t(768) << 20,
                      size_t(1) << 30, size_t(1536) << 20, N}) {
        for (int ns : {1, 2, 4}) {
            float best = 1e30f;
            for (int r = 0; r < 3; ++r) {
                CK(cudaDeviceSynchronize());
                CK(cudaEventRecord(a, s[0]));
                for (int k = 1; k < ns; ++k) CK(cudaStreamWaitEvent(s[k], a, 0));
                int i = 0;
                for (size_t o = 0; o < N; o += sz, ++i) {
                    size_t n = o + sz < N ? sz : N - o;
                    CK(cudaMemcpyAsync(h + o, d + o, n, cudaMemcpyDeviceToHost, s[i % ns]));
                }
                for (int k = 1; k < ns; ++k) {
                    CK(cudaEventRecord(j[k], s[k]));
                    CK(cudaStreamWaitEvent(s[0], j[k], 0));
                }
                CK(cudaEventRecord(b, s[0]));
                CK(cudaEventSynchronize(b));
                float ms;
                CK(cudaEventElapsedTime(&ms, a, b));
                if (ms < best) best = ms;
            }
            printf(" \"piece_%zuMB_streams_%d_GBps\": %.2f,\n", sz >> 20, ns, N / (best * 1e6));
        }
    }
    printf(" \"done\": 1\n}\n");
    return 0;
}
