// Launch-overhead probe: event-timed empty kernels of the fused kernel's shape
// (148 x 512 threads, 224 KB dynamic smem), cooperative or not, with or without
// a 256 MiB memset kernel before each (the bench's L2 flush).
#include <cstdio>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(512, 1) k_empty(int *p)
{
    extern __shared__ int s[];
    if (threadIdx.x == 0 && p) s[0] = blockIdx.x;
}

__global__ void k_fill(uint4 *p, size_t n)
{
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        p[i] = make_uint4(0, 0, 0, 0);
}

int main()
{
    const size_t SM = 224 * 1024;
    cudaFuncSetAttribute(k_empty, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SM);
    uint4 *buf;
    const size_t n = (256u << 20) / 16;
    cudaMalloc(&buf, n * 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int coop = 0; coop < 2; coop++)
        for (int flush = 0; flush < 2; flush++)
            for (size_t smem : {(size_t)0, SM}) {
                float tot = 0;
                for (int it = 0; it < 220; it++) {
                    if (flush) k_fill<<<592, 1024>>>(buf, n);
                    cudaLaunchConfig_t cfg = {};
                    cfg.gridDim = dim3(148);
                    cfg.blockDim = dim3(512);
                    cfg.dynamicSmemBytes = smem;
                    cudaLaunchAttribute a[1];
                    a[0].id = cudaLaunchAttributeCooperative;
                    a[0].val.cooperative = coop;
                    cfg.attrs = a;
                    cfg.numAttrs = 1;
                    cudaEventRecord(e0);
                    cudaLaunchKernelEx(&cfg, k_empty, (int *)nullptr);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms;
                    cudaEventElapsedTime(&ms, e0, e1);
                    if (it >= 20) tot += ms;
                }
                printf("coop=%d flush=%d smem=%zu: %.2f us per empty launch\n", coop, flush, smem,
                       tot / 200 * 1000);
            }
    // the same empty cooperative kernel as a one-node CUDA graph
    for (int flush = 0; flush < 2; flush++) {
        cudaStream_t st;
        cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
        cudaGraph_t g;
        cudaGraphExec_t ge;
        cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
        {
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(148);
            cfg.blockDim = dim3(512);
            cfg.dynamicSmemBytes = SM;
            cfg.stream = st;
            cudaLaunchAttribute a[1];
            a[0].id = cudaLaunchAttributeCooperative;
            a[0].val.cooperative = 1;
            cfg.attrs = a;
            cfg.numAttrs = 1;
            cudaLaunchKernelEx(&cfg, k_empty, (int *)nullptr);
        }
        cudaStreamEndCapture(st, &g);
        cudaGraphInstantiate(&ge, g, 0);
        float tot = 0;
        for (int it = 0; it < 220; it++) {
            if (flush) k_fill<<<592, 1024, 0, st>>>(buf, n);
            cudaEventRecord(e0, st);
            cudaGraphLaunch(ge, st);
            cudaEventRecord(e1, st);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (it >= 20) tot += ms;
        }
        printf("graph coop=1 flush=%d smem=%zu: %.2f us per empty launch\n", flush, SM, tot / 200 * 1000);
        // back-to-back events only (no kernel): the timing floor
        tot = 0;
        for (int it = 0; it < 220; it++) {
            if (flush) k_fill<<<592, 1024, 0, st>>>(buf, n);
            cudaEventRecord(e0, st);
            cudaEventRecord(e1, st);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (it >= 20) tot += ms;
        }
        printf("events only flush=%d: %.2f us\n", flush, tot / 200 * 1000);
    }
    return 0;
}
