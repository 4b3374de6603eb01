// Host build of device headers for CPU tests (tests/test_host_rr.py): the CUDA qualifiers become
// nothing and the few intrinsics the round-robin recurrence and its helpers use get plain C++
// definitions. Single-thread semantics only (warp functions act on one lane). Test infrastructure:
// the product library is always built by nvcc for sm_100a.
#pragma once
#define __CUDA_RUNTIME_H__
#include <cstdint>
#include <cstdio>
#include <cstring>
#define __device__
#define __host__
#define __global__
#define __shared__ static
#define __forceinline__ inline
#define __noinline__ __attribute__((noinline))
#define __restrict__
#define __launch_bounds__(...)
static inline int __popc(unsigned x){return __builtin_popcount(x);}
static inline int __popcll(unsigned long long x){return __builtin_popcountll(x);}
static inline int __ffs(int x){return __builtin_ffs(x);}
static inline int __ffsll(long long x){return __builtin_ffsll(x);}
static inline int __clz(int x){return x?__builtin_clz(x):32;}
static inline int __clzll(long long x){return x?__builtin_clzll(x):64;}
static inline unsigned __umulhi(unsigned a, unsigned b){return (unsigned)(((unsigned long long)a*b)>>32);}
static inline unsigned long long __umul64hi(unsigned long long a, unsigned long long b){return (unsigned long long)(((unsigned __int128)a*b)>>64);}
static inline unsigned __brev(unsigned x){unsigned r=0;for(int i=0;i<32;i++)if(x>>i&1)r|=1u<<(31-i);return r;}
static inline unsigned long long __brevll(unsigned long long x){unsigned long long r=0;for(int i=0;i<64;i++)if(x>>i&1)r|=1ull<<(63-i);return r;}
static inline unsigned __vcmpne4(unsigned a, unsigned b){unsigned r=0;for(int i=0;i<4;i++) if(((a>>(8*i))&255)!=((b>>(8*i))&255)) r|=255u<<(8*i); return r;}
static inline unsigned __byte_perm(unsigned x, unsigned y, unsigned s){unsigned long long v=((unsigned long long)y<<32)|x;unsigned r=0;for(int i=0;i<4;i++){unsigned sel=(s>>(4*i))&7;r|=((v>>(8*sel))&255)<<(8*i);}return r;}
struct uint4 {unsigned x,y,z,w;};
struct uint2 {unsigned x,y;};
struct dim3 {unsigned x,y,z;};
static dim3 threadIdx, blockIdx, blockDim, gridDim;
typedef void* cudaStream_t;
#define __align__(n) alignas(n)
struct ulonglong2 {unsigned long long x,y;};
struct ulonglong4 {unsigned long long x,y,z,w;};
static inline void __syncthreads(){}
static inline void __syncwarp(unsigned m=0xffffffffu){}
template<class T> static inline T __shfl_xor_sync(unsigned, T v, int, int=32){return v;}
template<class T> static inline T __shfl_sync(unsigned, T v, int, int=32){return v;}
template<class T> static inline T __shfl_up_sync(unsigned, T v, int, int=32){return v;}
template<class T> static inline T __shfl_down_sync(unsigned, T v, int, int=32){return v;}
static inline unsigned __activemask(){return 1;}
static inline int __all_sync(unsigned, int p){return p;}
static inline int __any_sync(unsigned, int p){return p;}
static inline unsigned __ballot_sync(unsigned, int p){return p?1:0;}
template<class T> static inline T __ldg(const T*p){return *p;}
static inline unsigned long long atomicMin(unsigned long long*p, unsigned long long v){auto o=*p; if(v<o)*p=v; return o;}
static inline unsigned atomicAdd(unsigned*p, unsigned v){auto o=*p; *p+=v; return o;}
static inline uint4 make_uint4(unsigned a,unsigned b,unsigned c,unsigned d){return uint4{a,b,c,d};}
#define VOP(name, op) static inline unsigned name(unsigned a, unsigned b){unsigned r=0;for(int i=0;i<4;i++){unsigned x=(a>>(8*i))&255,y=(b>>(8*i))&255; if(x op y) r|=255u<<(8*i);} return r;}
VOP(__vcmpgtu4, >) VOP(__vcmpeq4, ==) VOP(__vcmpltu4, <) VOP(__vcmpgeu4, >=) VOP(__vcmpleu4, <=)
