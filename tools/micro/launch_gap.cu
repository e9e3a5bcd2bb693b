// Launch-gap microbenchmark: back-to-back launches of a ~100 us kernel with a large parameter
// struct (like k_step's StepArgs), plain stream launches vs one CUDA graph of the same sequence.
#include <cstdio>
#include <cuda_runtime.h>
struct Big { double d[40]; long long i[8]; };
__global__ void k_spin(Big a, unsigned long long cycles, int* sink)
{
    const unsigned long long t0 = clock64();
    while (clock64() - t0 < cycles) { }
    if (a.i[0] == 12345 && threadIdx.x == 0) *sink = 1;
}
int main()
{
    int* sink; cudaMalloc(&sink, 4);
    cudaStream_t st; cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    Big b{}; cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int N = 2000;
    for (unsigned long long cyc : {0ull, 20000ull, 200000ull}) {
        for (int blocks : {148 * 6, 3907 + 3907 + 3907}) {
            k_spin<<<blocks, 256, 0, st>>>(b, cyc, sink);
            cudaStreamSynchronize(st);
            cudaEventRecord(e0, st);
            for (int i = 0; i < N; ++i) { b.i[1] = i; k_spin<<<blocks, 256, 0, st>>>(b, cyc, sink); }
            cudaEventRecord(e1, st); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            // graph of the same sequence
            cudaGraph_t g; cudaGraphExec_t ge;
            cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
            for (int i = 0; i < N; ++i) { b.i[1] = i; k_spin<<<blocks, 256, 0, st>>>(b, cyc, sink); }
            cudaStreamEndCapture(st, &g);
            cudaGraphInstantiate(&ge, g, 0);
            cudaGraphLaunch(ge, st); cudaStreamSynchronize(st);
            cudaEventRecord(e0, st); cudaGraphLaunch(ge, st); cudaEventRecord(e1, st); cudaEventSynchronize(e1);
            float msg; cudaEventElapsedTime(&msg, e0, e1);
            printf("spin %7llu cyc, %5d blocks: stream %7.2f us/launch, graph %7.2f us/launch\n", cyc, blocks, 1e3 * ms / N, 1e3 * msg / N);
            cudaGraphExecDestroy(ge); cudaGraphDestroy(g);
        }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
