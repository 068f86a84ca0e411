// PCIe paths for sptrsv_solve_host: how fast can 8 MB of b come in and 8 MB of x go out?
// (1) SM loads from pinned host memory (zero-copy), (2) SM stores to pinned host memory,
// (3) both at once, (4) copy-engine DMA H2D / D2H / both directions concurrently,
// (5) bulk (TMA-engine) copies host->smem.  CUDA events, best of 10.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_read(const double *__restrict__ h, double *__restrict__ d, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) d[i] = h[i];
}
__global__ void k_read2(const double2 *__restrict__ h, double2 *__restrict__ d, int n2) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n2) d[i] = h[i];
}
__global__ void k_write(const double *__restrict__ d, double *__restrict__ h, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) h[i] = d[i];
}
__global__ void k_write2(const double2 *__restrict__ d, double2 *__restrict__ h, int n2) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n2) h[i] = d[i];
}
__global__ void k_both(const double *__restrict__ hb, double *__restrict__ d, const double *__restrict__ d2,
                       double *__restrict__ hx, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) {
        d[i] = hb[i];
        hx[i] = d2[i];
    }
}
// one bulk copy of a CTA's 2 KB slice host -> smem, then smem -> device
__global__ void k_bulk(const double *__restrict__ h, double *__restrict__ d, int n) {
    __shared__ __align__(128) double s[256];
    __shared__ __align__(8) unsigned long long bar;
    const int r0 = blockIdx.x * 256;
    const int cnt = min(256, n - r0);
    unsigned sb = (unsigned)__cvta_generic_to_shared(&bar), ss = (unsigned)__cvta_generic_to_shared(s);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(sb));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(sb), "r"(cnt * 8));
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(ss), "l"(h + r0), "r"(cnt * 8), "r"(sb) : "memory");
    }
    asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared.b64 p, [%0], 0; @!p bra W; }" ::"r"(sb));
    if (threadIdx.x < cnt) d[r0 + threadIdx.x] = s[threadIdx.x];
}

int main() {
    const int n = 1000000;
    const size_t B = n * sizeof(double);
    double *hb, *hx, *d1, *d2;
    cudaHostAlloc(&hb, B, cudaHostAllocDefault);
    cudaHostAlloc(&hx, B, cudaHostAllocDefault);
    cudaMalloc(&d1, B);
    cudaMalloc(&d2, B);
    for (int i = 0; i < n; ++i) hb[i] = i;
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto run = [&](const char *name, double mb, auto f) {
        float best = 1e9;
        for (int r = 0; r < 10; ++r) {
            cudaEventRecord(e0, s1);
            f();
            cudaEventRecord(e1, s1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = ms < best ? ms : best;
        }
        printf("%-44s %8.1f us  %6.1f GB/s\n", name, best * 1e3, mb / (best * 1e-3) / 1e3);
    };
    const int g = (n + 255) / 256, g2 = (n / 2 + 255) / 256;
    run("SM loads from host (8 B/thread)", B / 1e6, [&] { k_read<<<g, 256, 0, s1>>>(hb, d1, n); });
    run("SM loads from host (16 B/thread)", B / 1e6, [&] { k_read2<<<g2, 256, 0, s1>>>((const double2 *)hb, (double2 *)d1, n / 2); });
    run("SM stores to host (8 B/thread)", B / 1e6, [&] { k_write<<<g, 256, 0, s1>>>(d2, hx, n); });
    run("SM stores to host (16 B/thread)", B / 1e6, [&] { k_write2<<<g2, 256, 0, s1>>>((const double2 *)d2, (double2 *)hx, n / 2); });
    run("SM loads + stores (both directions)", 2 * B / 1e6, [&] { k_both<<<g, 256, 0, s1>>>(hb, d1, d2, hx, n); });
    run("bulk copy host->smem per CTA (2 KB)", B / 1e6, [&] { k_bulk<<<g, 256, 0, s1>>>(hb, d1, n); });
    run("DMA H2D 8 MB", B / 1e6, [&] { cudaMemcpyAsync(d1, hb, B, cudaMemcpyHostToDevice, s1); });
    run("DMA D2H 8 MB", B / 1e6, [&] { cudaMemcpyAsync(hx, d2, B, cudaMemcpyDeviceToHost, s1); });
    run("DMA H2D + D2H concurrently (2 streams)", 2 * B / 1e6, [&] {
        cudaEvent_t f;
        cudaEventCreateWithFlags(&f, cudaEventDisableTiming);
        cudaEventRecord(f, s1);
        cudaStreamWaitEvent(s2, f, 0);
        cudaMemcpyAsync(d1, hb, B, cudaMemcpyHostToDevice, s1);
        cudaMemcpyAsync(hx, d2, B, cudaMemcpyDeviceToHost, s2);
        cudaEventRecord(f, s2);
        cudaStreamWaitEvent(s1, f, 0);
        cudaEventDestroy(f);
    });
    run("DMA H2D 16 x 512 KB chunks", B / 1e6, [&] {
        for (int c = 0; c < 16; ++c)
            cudaMemcpyAsync((char *)d1 + c * (B / 16), (char *)hb + c * (B / 16), B / 16, cudaMemcpyHostToDevice, s1);
    });
    printf("check %s\n", cudaGetLastError() == cudaSuccess ? "ok" : "CUDA error");
    return 0;
}
