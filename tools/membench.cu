// membench.cu — access-pattern microbenchmark for kernel A's HBM traffic:
// NR read streams + NW write streams of fp64 fields [nr][nt][np], either
// row-contiguous (like kernel B) or tiled (TJ x TK tile, march in r over a
// chunk of planes, like kernel A).  Prints GB/s (read+write bytes / time).
#include <cstdio>
#include <cuda_runtime.h>

template <int NR, int NW>
__global__ void rows_k(const double* __restrict__ in, double* __restrict__ out, long long N, int np,
                       int rows) {
    for (int row = blockIdx.x; row < rows; row += gridDim.x) {
        long long base = (long long)row * np;
        for (int k = 2 * threadIdx.x; k < np; k += 2 * blockDim.x) {
            double2 s = make_double2(0, 0);
#pragma unroll
            for (int f = 0; f < NR; f++) {
                double2 v = __ldg(reinterpret_cast<const double2*>(in + f * N + base + k));
                s.x += v.x; s.y += v.y;
            }
#pragma unroll
            for (int f = 0; f < NW; f++) *reinterpret_cast<double2*>(out + f * N + base + k) = s;
        }
    }
}

template <int NR, int NW, int TJ, int TK>
__global__ void tiles_k(const double* __restrict__ in, double* __restrict__ out, long long N, int nr,
                        int nt, int np, int chunk) {
    const int ntk = np / TK, ntj = nt / TJ;
    const int tk = blockIdx.x % ntk, tj = (blockIdx.x / ntk) % ntj, ch = blockIdx.x / (ntk * ntj);
    const int w = threadIdx.x / (TK / 2), l = threadIdx.x % (TK / 2);
    const long long off = (long long)(tj * TJ + w) * np + tk * TK + 2 * l;
    const long long plane = (long long)nt * np;
    for (int i = ch * chunk; i < min(nr, ch * chunk + chunk); i++) {
        const long long o = i * plane + off;
        double2 s = make_double2(0, 0);
#pragma unroll
        for (int f = 0; f < NR; f++) {
            double2 v = __ldg(reinterpret_cast<const double2*>(in + f * N + o));
            s.x += v.x; s.y += v.y;
        }
#pragma unroll
        for (int f = 0; f < NW; f++) *reinterpret_cast<double2*>(out + f * N + o) = s;
    }
}

int main() {
    const int nr = 256, nt = 256, np = 512;
    const long long N = (long long)nr * nt * np;
    constexpr int NR = 12, NW = 9;
    double *in, *out;
    cudaMalloc(&in, NR * N * 8);
    cudaMalloc(&out, NW * N * 8);
    cudaMemset(in, 0, NR * N * 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto run = [&](const char* name, auto launch) {
        for (int w = 0; w < 3; w++) launch();
        cudaEventRecord(a);
        for (int r = 0; r < 10; r++) launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        ms /= 10;
        printf("%-40s %.3f ms  %.0f GB/s\n", name, ms, (NR + NW) * N * 8 / (ms * 1e-3) / 1e9);
    };
    run("rows 256thr grid 148*8", [&] { rows_k<NR, NW><<<148 * 8, 256>>>(in, out, N, np, nr * nt); });
    run("tiles 8x64 chunk16", [&] { tiles_k<NR, NW, 8, 64><<<(nt / 8) * (np / 64) * (nr / 16), 256>>>(in, out, N, nr, nt, np, 16); });
    run("tiles 8x64 chunk32", [&] { tiles_k<NR, NW, 8, 64><<<(nt / 8) * (np / 64) * (nr / 32), 256>>>(in, out, N, nr, nt, np, 32); });
    run("tiles 4x128 chunk16", [&] { tiles_k<NR, NW, 4, 128><<<(nt / 4) * (np / 128) * (nr / 16), 256>>>(in, out, N, nr, nt, np, 16); });
    run("tiles 2x256 chunk16", [&] { tiles_k<NR, NW, 2, 256><<<(nt / 2) * (np / 256) * (nr / 16), 256>>>(in, out, N, nr, nt, np, 16); });
    run("tiles 1x512 chunk16", [&] { tiles_k<NR, NW, 1, 512><<<(nt / 1) * (np / 512) * (nr / 16), 256>>>(in, out, N, nr, nt, np, 16); });
    run("tiles 16x32 chunk16", [&] { tiles_k<NR, NW, 16, 32><<<(nt / 16) * (np / 32) * (nr / 16), 256>>>(in, out, N, nr, nt, np, 16); });
    run("tiles 8x64 chunk4", [&] { tiles_k<NR, NW, 8, 64><<<(nt / 8) * (np / 64) * (nr / 4), 256>>>(in, out, N, nr, nt, np, 4); });
    run("tiles 8x64 chunk1", [&] { tiles_k<NR, NW, 8, 64><<<(nt / 8) * (np / 64) * (nr / 1), 256>>>(in, out, N, nr, nt, np, 1); });
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
