// pipe_probe.cu -- issue throughput of the integer ops the hot loops use (IMAD, IMAD.HI, IMAD.IADD,
// IADD3, LOP3, PRMT, SHF, DP4A, LEA), full SM occupancy, 8 independent dependency chains per thread.
// Prints warp-instructions per cycle per SM for each op.  Build: nvcc -gencode
// arch=compute_100a,code=sm_100a -O3 -o tools/pipe_probe tools/pipe_probe.cu
#include <cstdio>
#include <cstdint>

#define N_ITER 4096
#define CH 8

template <int OP>
__device__ __forceinline__ uint32_t op(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    if constexpr (OP == 0) asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    if constexpr (OP == 1) asm volatile("mad.hi.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    if constexpr (OP == 2) asm volatile("add.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(c));
    if constexpr (OP == 3) asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    if constexpr (OP == 4) asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(c), "r"(b));
    if constexpr (OP == 5) asm volatile("shf.r.wrap.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(c), "r"(b));
    if constexpr (OP == 6) asm volatile("dp4a.u32.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    if constexpr (OP == 7) asm volatile("add.u32 %0, %1, %2; add.u32 %0, %0, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    if constexpr (OP == 8) asm volatile("{ .reg .pred p; setp.ge.u32 p, %1, %2; selp.u32 %0, 1, 0, p; }" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

template <int OP>
__global__ void probe(uint32_t *out, uint32_t b, long long *cyc)
{
    uint32_t x[CH];
#pragma unroll
    for (int i = 0; i < CH; i++) x[i] = threadIdx.x * 7 + i;
    __syncthreads();
    long long t0 = clock64();
    for (int it = 0; it < N_ITER; it++) {
#pragma unroll
        for (int i = 0; i < CH; i++) x[i] = op<OP>(x[i], b, x[(i + 1) % CH]);
    }
    __syncthreads();
    long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < CH; i++) s ^= x[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char *name, uint32_t *out, long long *cyc)
{
    const int threads = 1024, blocks = 148;
    probe<OP><<<blocks, threads>>>(out, 0x01010101u, cyc);
    cudaDeviceSynchronize();
    probe<OP><<<blocks, threads>>>(out, 0x01010101u, cyc);
    cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < blocks; i++) avg += h[i];
    avg /= blocks;
    const double winst = (double)(threads / 32) * N_ITER * CH;  // warp-instructions per SM (of the op)
    printf("%-12s %.3f warp-inst/cycle/SM  (%.2f cycles per warp-inst per SMSP)\n", name, winst / avg,
           4.0 * avg / winst);
}

int main()
{
    uint32_t *out;
    long long *cyc;
    cudaMalloc(&out, 148 * 1024 * 4);
    cudaMalloc(&cyc, 148 * 8);
    run<0>("IMAD", out, cyc);
    run<1>("IMAD.HI", out, cyc);
    run<2>("IADD", out, cyc);
    run<3>("LOP3", out, cyc);
    run<4>("PRMT", out, cyc);
    run<5>("SHF.R.W", out, cyc);
    run<6>("DP4A", out, cyc);
    run<7>("IADD x2", out, cyc);
    run<8>("ISETP+SEL", out, cyc);
    return 0;
}
