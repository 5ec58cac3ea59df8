// Link micro-benchmark (§III-B: "B_ij ... can be evaluated via micro benchmark"): read, write
// and random-atomic throughput and dependent-load latency of device `exec` on memory of device `mem` (a peer
// over NVLink 5 / NVSwitch when they differ, local HBM when equal). Measurement tool only -- not on the hot
// path; tools/nvlink_bench.py drives it and derives the FSteal remote cost c_ij = B_local / B_ij.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

namespace {

__global__ void k_read(const uint4* __restrict__ p, size_t n, unsigned long long* sink) {
    uint4 acc = make_uint4(0, 0, 0, 0);
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        const uint4 v = __ldcs(p + i);
        acc.x ^= v.x;
        acc.y ^= v.y;
        acc.z ^= v.z;
        acc.w ^= v.w;
    }
    if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x9E3779B9u) atomicAdd(sink, 1ull);  // keeps the loads alive
}

__global__ void k_write(uint4* __restrict__ p, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        __stcs(p + i, make_uint4((unsigned)i, 1u, 2u, 3u));
}

__global__ void k_atomic(unsigned* p, unsigned long long words, unsigned long long ops) {
    unsigned long long x = 0x9E3779B97F4A7C15ull * (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x + 1);
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < ops;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        x ^= x >> 12;
        x ^= x << 25;
        x ^= x >> 27;
        atomicAdd(p + (x * 0x2545F4914F6CDD1Dull >> 20) % words, 1u);  // RED.ADD (no return)
    }
}

__global__ void k_init_chase(unsigned* p, unsigned n, unsigned stride) {
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        p[i] = (unsigned)(((unsigned long long)i + stride) % n);
}

__global__ void k_chase(const unsigned* p, unsigned steps, unsigned* out) {
    unsigned j = 0;
    for (unsigned s = 0; s < steps; s++) j = __ldcg(p + j);
    *out = j;
}

int enable_peer(int exec, int mem) {
    if (exec == mem) return 0;
    int can = 0;
    cudaDeviceCanAccessPeer(&can, exec, mem);
    if (!can) return -1;
    cudaSetDevice(exec);
    cudaError_t e = cudaDeviceEnablePeerAccess(mem, 0);
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return -2;
    cudaGetLastError();
    return 0;
}

}  // namespace

extern "C" {

int lb_device_count(void) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) return 0;
    return n;
}

// GB/s of device `exec` streaming `bytes` from (read = 1) or to (read = 0) memory on device `mem`.
int lb_stream_bw(int exec, int mem, unsigned long long bytes, int reps, int read, double* gbps) {
    if (enable_peer(exec, mem)) return -1;
    cudaSetDevice(mem);
    void* buf = nullptr;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) return -2;
    cudaMemset(buf, 1, bytes);
    cudaDeviceSynchronize();
    cudaSetDevice(exec);
    unsigned long long* sink = nullptr;
    cudaMalloc(&sink, 8);
    int nsm = 148;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, exec);
    const size_t n = bytes / 16;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int w = 0; w < 2; w++) read ? k_read<<<nsm * 8, 512>>>((const uint4*)buf, n, sink) : k_write<<<nsm * 8, 512>>>((uint4*)buf, n);
    cudaEventRecord(a);
    for (int r = 0; r < reps; r++) read ? k_read<<<nsm * 8, 512>>>((const uint4*)buf, n, sink) : k_write<<<nsm * 8, 512>>>((uint4*)buf, n);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    *gbps = (double)bytes * reps / (ms / 1e3) / 1e9;
    const cudaError_t e = cudaGetLastError();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(sink);
    cudaSetDevice(mem);
    cudaFree(buf);
    return e == cudaSuccess ? 0 : -3;
}

// Giga random 4-byte atomics (red.add) per second of device `exec` into a 256 MB buffer on device `mem`.
int lb_atomic_rate(int exec, int mem, unsigned long long ops, double* gops) {
    if (enable_peer(exec, mem)) return -1;
    const unsigned long long words = 64ull << 20;
    cudaSetDevice(mem);
    unsigned* buf = nullptr;
    if (cudaMalloc(&buf, words * 4) != cudaSuccess) return -2;
    cudaMemset(buf, 0, words * 4);
    cudaDeviceSynchronize();
    cudaSetDevice(exec);
    int nsm = 148;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, exec);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    k_atomic<<<nsm * 8, 512>>>(buf, words, ops / 8);
    cudaEventRecord(a);
    k_atomic<<<nsm * 8, 512>>>(buf, words, ops);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    *gops = (double)ops / (ms / 1e3) / 1e9;
    const cudaError_t e = cudaGetLastError();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaSetDevice(mem);
    cudaFree(buf);
    return e == cudaSuccess ? 0 : -3;
}

// Dependent-load latency (ns) of device `exec` on memory of device `mem`: a single-thread pointer chase with
// a large stride over a 1 GB array (beyond L2).
int lb_latency(int exec, int mem, unsigned steps, double* ns) {
    if (enable_peer(exec, mem)) return -1;
    const unsigned n = 1u << 28;
    cudaSetDevice(mem);
    unsigned* buf = nullptr;
    if (cudaMalloc(&buf, (size_t)n * 4) != cudaSuccess) return -2;
    k_init_chase<<<1184, 256>>>(buf, n, 1000003u * 8u + 33u);
    cudaDeviceSynchronize();
    cudaSetDevice(exec);
    unsigned* out = nullptr;
    cudaMalloc(&out, 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    k_chase<<<1, 1>>>(buf, 1000, out);
    cudaEventRecord(a);
    k_chase<<<1, 1>>>(buf, steps, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    *ns = (double)ms * 1e6 / steps;
    const cudaError_t e = cudaGetLastError();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(out);
    cudaSetDevice(mem);
    cudaFree(buf);
    return e == cudaSuccess ? 0 : -3;
}

}  // extern "C"
