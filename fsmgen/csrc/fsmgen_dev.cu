// fsmgen_dev.cu -- device twin of fsmgen.c: fills device memory with the same counter-based
// SplitMix64 byte stream, so that a 64 GiB input (config C5) can be generated in place in HBM
// while the oracle side regenerates identical bytes on the host with fsmgen.c.
// Workload generator only: no spec-k arithmetic here.
#include <cstdint>
#include <cuda_runtime.h>

namespace {
constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ULL;

__device__ __forceinline__ uint64_t mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

// out is 8-byte aligned at stream byte `offset` (offset % 8 == 0); writes n_words whole words.
__global__ void fill_words(uint64_t *__restrict__ out, uint64_t seed, uint64_t word0, uint64_t n_words)
{
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_words; i += stride)
        out[i] = mix64(seed + (word0 + i + 1) * kGolden);
}

// byte-granular fill for unaligned heads/tails
__global__ void fill_bytes(uint8_t *__restrict__ out, uint64_t seed, uint64_t offset, uint64_t len)
{
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += stride) {
        uint64_t j = offset + i;
        out[i] = (uint8_t)(mix64(seed + ((j >> 3) + 1) * kGolden) >> (8 * (j & 7)));
    }
}
// Measurement helper: a read-only streaming kernel over the same input -- 32-byte
// non-coherent loads, 4 in flight per thread, XOR-folded into one word per thread so nothing is
// elided.  Its GB/s is the achievable HBM *read* ceiling the FSM kernel is compared against (the
// MEASURED_PEAKS figure is a copy, read + write).
__global__ void read_stream(const uint8_t *__restrict__ in, uint64_t n32, uint32_t *__restrict__ sink)
{
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (; i + 3 * stride < n32; i += 4 * stride) {
        uint32_t v[4][8];
#pragma unroll
        for (int u = 0; u < 4; u++)
            asm volatile("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(v[u][0]), "=r"(v[u][1]), "=r"(v[u][2]), "=r"(v[u][3]), "=r"(v[u][4]),
                           "=r"(v[u][5]), "=r"(v[u][6]), "=r"(v[u][7])
                         : "l"(in + 32 * (i + u * stride)));
#pragma unroll
        for (int u = 0; u < 4; u++)
#pragma unroll
            for (int w = 0; w < 8; w++) acc ^= v[u][w];
    }
    for (; i < n32; i += stride) {
        const uint4 *q = reinterpret_cast<const uint4 *>(in + 32 * i);
        const uint4 a = __ldg(q), b = __ldg(q + 1);
        acc ^= a.x ^ a.y ^ a.z ^ a.w ^ b.x ^ b.y ^ b.z ^ b.w;
    }
    if (acc == 0x9E3779B9u) sink[0] = acc;  // practically never taken; keeps the loads live
}
} // namespace

// Read-only streaming pass over n bytes (32-byte aligned pointer, n multiple of 32 used).
extern "C" int fsmgen_dev_read_stream(const void *dev_in, uint64_t n, void *dev_sink, int num_sms, void *stream)
{
    const uint64_t n32 = n / 32;
    read_stream<<<num_sms * 8, 256, 0, (cudaStream_t)stream>>>((const uint8_t *)dev_in, n32, (uint32_t *)dev_sink);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

extern "C" int fsmgen_dev_fill(void *dev_out, uint64_t seed, uint64_t offset, uint64_t len, void *stream)
{
    cudaStream_t s = (cudaStream_t)stream;
    uint8_t *out = (uint8_t *)dev_out;
    if (len == 0) return 0;
    // Whole words only where both the stream position and the pointer are 8-aligned.
    uint64_t head = (8 - (offset & 7)) & 7;
    if (head > len) head = len;
    if (head) fill_bytes<<<1, 64, 0, s>>>(out, seed, offset, head);
    uint64_t rest = len - head, pos = offset + head;
    uint8_t *p = out + head;
    if (((uintptr_t)p & 7) == 0) {
        uint64_t nw = rest >> 3;
        if (nw) fill_words<<<148 * 8, 256, 0, s>>>((uint64_t *)p, seed, pos >> 3, nw);
        uint64_t tail = rest & 7;
        if (tail) fill_bytes<<<1, 64, 0, s>>>(p + (nw << 3), seed, pos + (nw << 3), tail);
    } else if (rest) {
        fill_bytes<<<148 * 8, 256, 0, s>>>(p, seed, pos, rest);
    }
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
