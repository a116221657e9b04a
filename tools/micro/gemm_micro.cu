// Standalone latency microbenchmark of the small-GEMM kernel variants on the MLP's Beaver shapes
// (warm, in a CUDA graph of R launches).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
// -std=c++17 -I.. gemm_micro.cu -o gemm_micro
#include <cstdio>
#include <vector>
#include "../../paper_conf_icpp_chenzzzz020_b200/csrc/gemm_simt.cuh"

namespace psml {
psml_status fail(psml_status s, const std::string &m) { fprintf(stderr, "%s\n", m.c_str()); return s; }
}  // namespace psml
using namespace psml;
using T = uint64_t;

__global__ void fill(T *p, int64_t n, uint64_t s) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = (i + 1) * 0x9E3779B97F4A7C15ull ^ s;
}

int main(int argc, char **argv) {
    const bool prof = argc > 1;
    struct S { int64_t M, K, N; };
    std::vector<S> shapes = {{128, 784, 128}, {128, 128, 128}, {128, 128, 10}, {128, 10, 128}, {784, 128, 128}};
    const int R = 50;
    for (auto sh : shapes) {
        const int64_t M = sh.M, K = sh.K, N = sh.N;
        T *buf;
        const int64_t words = 4 * M * K + 4 * K * N + 4 * M * N + 2 * M * N;
        cudaMalloc(&buf, words * 8);
        fill<<<1024, 256>>>(buf, words, 7);
        BeaverOps<T, 0> ops{};
        T *q = buf;
        ops.mE0 = q; q += M * K; ops.mE1 = q; q += M * K;
        ops.U[0] = q; q += M * K; ops.U[1] = q; q += M * K;
        ops.mF0 = q; q += K * N; ops.mF1 = q; q += K * N;
        ops.V[0] = q; q += K * N; ops.V[1] = q; q += K * N;
        ops.Z[0] = q; q += M * N; ops.Z[1] = q; q += M * N;
        ops.C[0] = q; q += M * N; ops.C[1] = q; q += M * N;
        T *ws = q;
        ops.M = M; ops.N = N; ops.K = K; ops.Kext = 2 * K; ops.trunc = 13;
        cudaStream_t s;
        cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
        auto timeit = [&](const char *name, auto launch) {
            cudaGraph_t g;
            cudaGraphExec_t ge;
            cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
            for (int r = 0; r < R; ++r) launch();
            cudaStreamEndCapture(s, &g);
            cudaGraphInstantiate(&ge, g, 0);
            cudaGraphLaunch(ge, s);
            cudaStreamSynchronize(s);
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            cudaEventRecord(e0, s);
            for (int i = 0; i < 10; ++i) cudaGraphLaunch(ge, s);
            cudaEventRecord(e1, s);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("%lldx%lldx%lld %-14s %8.2f us  (%s)\n", (long long)M, (long long)K, (long long)N, name,
                   ms * 1e3 / (10 * R), cudaGetErrorString(cudaGetLastError()));
            cudaGraphExecDestroy(ge);
            cudaGraphDestroy(g);
        };
        using Op = BeaverOps<T, 0>;
        if (prof) {   // plain launches for ncu
            for (int i = 0; i < 3; ++i) launch_ring_gemm_cl<T, Op, ClCfg<32, 32, 256, 2, 2>>(ops, s, 148, 8);
            cudaStreamSynchronize(s);
            cudaFree(buf);
            continue;
        }
        timeit("small", [&] {
            dim3 grid((unsigned)((N + 15) / 16), (unsigned)((M + 15) / 16), 2);
            ring_gemm_small<T, Op><<<grid, 256, 0, s>>>(ops, 2 * K, nullptr);
        });
        timeit("cl32x32/128", [&] { launch_ring_gemm_cl<T, Op, ClDefault>(ops, s, 148, 8); });
        timeit("cl32x32/256", [&] { launch_ring_gemm_cl<T, Op, ClCfg<32, 32, 256, 2, 2>>(ops, s, 148, 8); });
        timeit("cl32x32/256k4", [&] { launch_ring_gemm_cl<T, Op, ClCfg<32, 32, 256, 2, 2>>(ops, s, 148, 4); });
        timeit("cl64x32/256b16", [&] { launch_ring_gemm_cl<T, Op, ClCfg<64, 32, 256, 2, 4, 16>>(ops, s, 148, 8); });
        timeit("cl32x64/256b16", [&] { launch_ring_gemm_cl<T, Op, ClCfg<32, 64, 256, 2, 4, 16>>(ops, s, 148, 8); });
        timeit("cl32x32/128b16", [&] { launch_ring_gemm_cl<T, Op, ClCfg<32, 32, 128, 2, 4, 16>>(ops, s, 148, 8); });
        timeit("cl32x32/256b16", [&] { launch_ring_gemm_cl<T, Op, ClCfg<32, 32, 256, 2, 2, 16>>(ops, s, 148, 8); });
        timeit("cl16x32/128", [&] { launch_ring_gemm_cl<T, Op, ClCfg<16, 32, 128, 2, 2>>(ops, s, 148, 8); });
        cudaFree(buf);
    }
    return 0;
}
