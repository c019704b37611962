// Hardware probe (not part of the product path): FP64 pipe throughput on sm_100a.
// Measures DFMA (vector) and DMMA (mma.sync .f64) issue throughput so the tile
// kernel design (SURVEY.md §0.1, §7 "hard parts") is chosen by measurement.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("ERR %s @%d: %s\n",#x,__LINE__,cudaGetErrorString(e)); return 1;}}while(0)

template<int ILP>
__global__ void dfma_loop(double* out, int iters, double a, double b){
  double acc[ILP];
  #pragma unroll
  for(int i=0;i<ILP;i++) acc[i]=threadIdx.x*1e-3+i;
  for(int it=0; it<iters; ++it){
    #pragma unroll
    for(int i=0;i<ILP;i++) acc[i]=fma(acc[i],a,b);
  }
  double s=0;
  #pragma unroll
  for(int i=0;i<ILP;i++) s+=acc[i];
  if(s==1234.5) out[threadIdx.x]=s;
}

template<int ILP>
__global__ void dmma884_loop(double* out, int iters){
  double a = 1.0 + threadIdx.x*1e-6, b = 0.999;
  double c[ILP][2];
  #pragma unroll
  for(int i=0;i<ILP;i++){c[i][0]=0;c[i][1]=0;}
  for(int it=0; it<iters; ++it){
    #pragma unroll
    for(int i=0;i<ILP;i++){
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
        : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
  }
  double s=0;
  #pragma unroll
  for(int i=0;i<ILP;i++) s+=c[i][0]+c[i][1];
  if(s==1234.5) out[threadIdx.x]=s;
}

template<int ILP>
__global__ void dmma16816_loop(double* out, int iters){
  double a[8], b[4];
  #pragma unroll
  for(int i=0;i<8;i++) a[i]=1.0+i*1e-7;
  #pragma unroll
  for(int i=0;i<4;i++) b[i]=0.999;
  double c[ILP][4];
  #pragma unroll
  for(int i=0;i<ILP;i++){c[i][0]=c[i][1]=c[i][2]=c[i][3]=0;}
  for(int it=0; it<iters; ++it){
    #pragma unroll
    for(int i=0;i<ILP;i++){
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};\n"
        : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3])
        : "d"(a[0]),"d"(a[1]),"d"(a[2]),"d"(a[3]),"d"(a[4]),"d"(a[5]),"d"(a[6]),"d"(a[7]),
          "d"(b[0]),"d"(b[1]),"d"(b[2]),"d"(b[3]));
    }
  }
  double s=0;
  #pragma unroll
  for(int i=0;i<ILP;i++) s+=c[i][0]+c[i][1]+c[i][2]+c[i][3];
  if(s==1234.5) out[threadIdx.x]=s;
}

template<typename K>
float timeit(K k, int blocks, int threads, int reps=5){
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k(); cudaDeviceSynchronize();
  float best=1e30f;
  for(int r=0;r<reps;r++){
    cudaEventRecord(e0); k(); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms,e0,e1); if(ms<best) best=ms;
  }
  return best;
}

int main(){
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,0));
  int clk=0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("device %s SMs %d cc %d.%d clockRate(kHz) %d smemPerBlockOptin %zu l2 %d regsPerSM %d\n",
    p.name, p.multiProcessorCount, p.major, p.minor, clk, p.sharedMemPerBlockOptin, p.l2CacheSize, p.regsPerMultiprocessor);
  double* out; CK(cudaMalloc(&out, 4096*8));
  int SM=p.multiProcessorCount;
  int iters=20000;
  for(int w: {4,8,16}){
    int thr=32*w;
    float ms=timeit([&]{dfma_loop<8><<<SM*2,thr>>>(out,iters,1.0000001,1e-9);}, 0,0);
    double fl=2.0*8*iters*(double)thr*SM*2;
    printf("DFMA ilp8 warps/cta %d x2cta: %.3f ms  %.2f TFLOP/s\n", w, ms, fl/ms/1e9);
  }
  for(int w: {4,8,16}){
    int thr=32*w;
    float ms=timeit([&]{dmma884_loop<8><<<SM*2,thr>>>(out,iters/4);}, 0,0);
    double fl=2.0*256*8*(iters/4)*(double)(thr/32)*SM*2;
    printf("DMMA m8n8k4 ilp8 warps/cta %d x2cta: %.3f ms  %.2f TFLOP/s\n", w, ms, fl/ms/1e9);
  }
  for(int w: {4,8}){
    int thr=32*w;
    float ms=timeit([&]{dmma16816_loop<4><<<SM*2,thr>>>(out,iters/32);}, 0,0);
    double fl=2.0*16*8*16*4*(iters/32)*(double)(thr/32)*SM*2;
    printf("DMMA m16n8k16 ilp4 warps/cta %d x2cta: %.3f ms  %.2f TFLOP/s\n", w, ms, fl/ms/1e9);
  }
  return 0;
}
