#include <cstdio>
#include <cstdint>
extern __shared__ uint8_t dsm[];
__global__ void k(uint32_t* o){ if(threadIdx.x==0){ o[0]=(uint32_t)__cvta_generic_to_shared(dsm);} }
__global__ void k2(uint32_t* o){ __shared__ uint32_t st[4]; st[threadIdx.x&3]=1; __syncthreads(); if(threadIdx.x==0){ o[1]=(uint32_t)__cvta_generic_to_shared(dsm); o[2]=(uint32_t)__cvta_generic_to_shared(st);} }
int main(){ uint32_t* d; cudaMalloc(&d,16); cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
 k<<<1,32,100000>>>(d); k2<<<1,32,1000>>>(d); uint32_t h[4]; cudaMemcpy(h,d,16,cudaMemcpyDeviceToHost); printf("dyn-only base=%u  dyn-with-static base=%u static=%u\n",h[0],h[1],h[2]); return 0;}
