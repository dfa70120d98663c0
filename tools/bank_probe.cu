// Microbenchmark: how does sm_100 group the 32 lanes of a 128-bit shared load
// into bank-conflict phases?  Each kernel variant loads float4 sm[idx(lane)];
// run under ncu and read l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum.
#include <cstdio>
#include <cuda_runtime.h>

template <int V>
__global__ void probe(float* out) {
    __shared__ float4 sm[512];
    for (int i = threadIdx.x; i < 512; i += blockDim.x) sm[i] = make_float4(i, i, i, i);
    __syncthreads();
    const int l = threadIdx.x & 31;
    int idx;
    if (V == 0) idx = l;                          // contiguous: ideal
    else if (V == 1) idx = (l & 7) * 8;           // lanes 0-7 same residue, distinct addresses; l and l+8 equal
    else if (V == 2) idx = l * 8;                 // all 32 lanes residue 0, distinct addresses
    else if (V == 3) idx = (l >> 2) * 8 + (l & 3) * 64;  // residue 0 everywhere, groups of 4
    else if (V == 4) idx = (l & 7) + 8 * (l >> 3) * 8;   // within each group of 8 consecutive lanes distinct residues
    else if (V == 5) idx = ((l >> 3) + 4 * (l & 7)) ;    // strided grouping test: lanes l, l+8, l+16, l+24 distinct residues?
    else idx = (l % 4) * 8 + (l / 4);             // residues distinct among lanes {4k..4k+3}?
    float acc = 0.f;
#pragma unroll 1
    for (int it = 0; it < 64; ++it) {
        const float4 v = sm[(idx + it * 0) & 511];
        acc += v.x + v.y;
    }
    if (acc == -1.f) out[threadIdx.x] = acc;
}

int main() {
    float* o;
    cudaMalloc(&o, 1024 * 4);
    probe<0><<<1, 32>>>(o);
    probe<1><<<1, 32>>>(o);
    probe<2><<<1, 32>>>(o);
    probe<3><<<1, 32>>>(o);
    probe<4><<<1, 32>>>(o);
    probe<5><<<1, 32>>>(o);
    probe<6><<<1, 32>>>(o);
    cudaDeviceSynchronize();
    printf("done\n");
    return 0;
}
