// Are the packed f32x2 instructions bit-identical to their scalar forms on sm_100a?
// Compares __ffma2_rn / __fadd2_rn / __fmul2_rn with fmaf / __fadd_rn / __fmul_rn on random inputs.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t mix(uint64_t z){z+=0x9e3779b97f4a7c15ull;z=(z^(z>>30))*0xbf58476d1ce4e5b9ull;z=(z^(z>>27))*0x94d049bb133111ebull;return z^(z>>31);}
__device__ float rnd(uint64_t k, int mode){
  uint64_t z=mix(k); float u=(float)(z>>40)*(1.0f/16777216.0f);
  if(mode==0) return u*8.f-4.f;                       // Sobel-range values
  if(mode==1) return ldexpf(u+0.5f,(int)(mix(k^7)%60)-40) * ((z&1)?-1.f:1.f);  // wide exponents
  return u;
}
__global__ void k(unsigned long long *bad, int mode){
  uint64_t i = blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;
  float a=rnd(3*i,mode), b=rnd(3*i+1,mode), c=rnd(3*i+2,mode), d=rnd(3*i+3,mode), e=rnd(3*i+4,mode), f=rnd(3*i+5,mode);
  float2 r=__ffma2_rn(make_float2(a,d),make_float2(b,e),make_float2(c,f));
  if(__float_as_uint(r.x)!=__float_as_uint(__fmaf_rn(a,b,c))||__float_as_uint(r.y)!=__float_as_uint(__fmaf_rn(d,e,f))) atomicAdd(bad+0,1ull);
  float2 s=__fadd2_rn(make_float2(a,d),make_float2(b,e));
  if(__float_as_uint(s.x)!=__float_as_uint(__fadd_rn(a,b))||__float_as_uint(s.y)!=__float_as_uint(__fadd_rn(d,e))) atomicAdd(bad+1,1ull);
  float2 m=__fmul2_rn(make_float2(a,d),make_float2(b,e));
  if(__float_as_uint(m.x)!=__float_as_uint(__fmul_rn(a,b))||__float_as_uint(m.y)!=__float_as_uint(__fmul_rn(d,e))) atomicAdd(bad+2,1ull);
  // fma with a product operand: fma(a*b, c, d) vs f32x2
  float p=__fmul_rn(a,b), q=__fmul_rn(d,e);
  float2 t=__ffma2_rn(make_float2(-p,-q),make_float2(c,f),make_float2(a,d));
  if(__float_as_uint(t.x)!=__float_as_uint(__fmaf_rn(-p,c,a))||__float_as_uint(t.y)!=__float_as_uint(__fmaf_rn(-q,f,d))) atomicAdd(bad+3,1ull);
}
int main(){
  unsigned long long *d,h[4];
  cudaMalloc(&d,32);
  for(int mode=0;mode<3;mode++){
    cudaMemset(d,0,32);
    k<<<1<<16,256>>>(d,mode);
    cudaMemcpy(h,d,32,cudaMemcpyDeviceToHost);
    printf("mode %d of %d: ffma2 %llu fadd2 %llu fmul2 %llu nfma2 %llu mismatches\n",mode,1<<24,h[0],h[1],h[2],h[3]);
  }
  return 0;
}
