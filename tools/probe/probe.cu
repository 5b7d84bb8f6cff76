// Box probe: launch cost, stream-memop cost, priorities, green contexts (one-off measurement tool).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <chrono>
#include <vector>
#include <set>
#include <algorithm>
#include <dlfcn.h>
#define CK(x) do{auto e=(x); if(e!=cudaSuccess){printf("ERR %s:%d %s\n",__FILE__,__LINE__,cudaGetErrorString(e));return 1;}}while(0)
#define CD(x) do{CUresult e=(x); if(e!=CUDA_SUCCESS){const char*s;cuGetErrorString(e,&s);printf("DRV ERR %s:%d %s\n",__FILE__,__LINE__,s);}}while(0)
__global__ void empty_k(int*) {}
__global__ void smid_k(int* out, long spin) {
  unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  if (threadIdx.x==0) out[blockIdx.x] = s;
  long t0 = clock64(); while (clock64()-t0 < spin) {}
}
static double now_us(){return std::chrono::duration<double,std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();}
int main(){
  CK(cudaSetDevice(0)); CK(cudaFree(0));
  int lo,hi; CK(cudaDeviceGetStreamPriorityRange(&lo,&hi)); printf("prio range least=%d greatest=%d\n",lo,hi);
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0); printf("SMs %d\n", nsm);
  cudaStream_t s; CK(cudaStreamCreateWithPriority(&s, cudaStreamNonBlocking, hi));
  int* d; CK(cudaMalloc(&d, 4096*4));
  for(int i=0;i<1000;i++) empty_k<<<1,32,0,s>>>(d);
  CK(cudaStreamSynchronize(s));
  int N=20000; double t0=now_us(); for(int i=0;i<N;i++) empty_k<<<1,32,0,s>>>(d); double t1=now_us();
  CK(cudaStreamSynchronize(s)); double t2=now_us();
  printf("runtime <<<>>> launch: %.3f us/launch CPU, %.3f us/launch end-to-end\n",(t1-t0)/N,(t2-t0)/N);
  cudaKernel_t kk; CK(cudaGetKernel(&kk, (const void*)empty_k));
  void* args[] = {&d};
  t0=now_us(); for(int i=0;i<N;i++) CD(cuLaunchKernel((CUfunction)kk,1,1,1,32,1,1,0,(CUstream)s,args,nullptr)); t1=now_us();
  CK(cudaStreamSynchronize(s)); t2=now_us();
  printf("cuLaunchKernel(CUkernel): %.3f us/launch CPU, %.3f e2e\n",(t1-t0)/N,(t2-t0)/N);
  CUfunction f; CD(cuKernelGetFunction(&f,(CUkernel)kk));
  t0=now_us(); for(int i=0;i<N;i++) CD(cuLaunchKernel(f,1,1,1,32,1,1,0,(CUstream)s,args,nullptr)); t1=now_us();
  CK(cudaStreamSynchronize(s)); t2=now_us();
  printf("cuLaunchKernel(CUfunction): %.3f us/launch CPU, %.3f e2e\n",(t1-t0)/N,(t2-t0)/N);
  // stream write value
  unsigned long long* hc; CK(cudaHostAlloc(&hc, 64, cudaHostAllocMapped)); *hc=0;
  CUdeviceptr dc; CD(cuMemHostGetDevicePointer(&dc, hc, 0));
  t0=now_us(); for(int i=0;i<N;i++) CD(cuStreamWriteValue64((CUstream)s, dc, i+1, 0)); t1=now_us();
  CK(cudaStreamSynchronize(s));
  printf("cuStreamWriteValue64: %.3f us/op CPU; final=%llu\n",(t1-t0)/N,*(volatile unsigned long long*)hc);
  t0=now_us(); for(int i=0;i<N;i++){ CD(cuLaunchKernel(f,1,1,1,32,1,1,0,(CUstream)s,args,nullptr)); CD(cuStreamWriteValue64((CUstream)s, dc, N+i+1, 0));} t1=now_us();
  CK(cudaStreamSynchronize(s)); printf("launch+write: %.3f us/pair CPU\n",(t1-t0)/N);
  // round trip: launch + write, spin until seen
  std::vector<double> rt;
  for(int i=0;i<2000;i++){ double a=now_us(); CD(cuLaunchKernel(f,1,1,1,32,1,1,0,(CUstream)s,args,nullptr)); CD(cuStreamWriteValue64((CUstream)s, dc, 10*N+i, 0));
    while(*(volatile unsigned long long*)hc != (unsigned long long)(10*N+i)){} rt.push_back(now_us()-a);}
  std::sort(rt.begin(),rt.end()); printf("launch->host-visible completion: p50 %.2f us p99 %.2f us\n", rt[1000], rt[1980]);
  // events
  cudaEvent_t ev; CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  t0=now_us(); for(int i=0;i<N;i++) CK(cudaEventRecord(ev,s)); t1=now_us(); CK(cudaStreamSynchronize(s));
  printf("cudaEventRecord: %.3f us\n",(t1-t0)/N);
  t0=now_us(); for(int i=0;i<N;i++) cudaEventQuery(ev); t1=now_us(); printf("cudaEventQuery: %.3f us\n",(t1-t0)/N);
  // green contexts
  CUdevice dev; CD(cuDeviceGet(&dev,0));
  CUdevResource all; CD(cuDeviceGetDevResource(dev,&all,CU_DEV_RESOURCE_TYPE_SM)); printf("green: device SM resource %u\n", all.sm.smCount);
  for (unsigned want : {8u, 32u, 64u, 72u, 140u}) {
    CUdevResource part[2]; unsigned n=1; CUdevResource rem;
    CD(cuDevSmResourceSplitByCount(part,&n,&all,&rem,0,want));
    CUdevResourceDesc desc; CD(cuDevResourceGenerateDesc(&desc,&part[0],1));
    CUgreenCtx g; CD(cuGreenCtxCreate(&g,desc,dev,CU_GREEN_CTX_DEFAULT_STREAM));
    CUstream gs; CD(cuGreenCtxStreamCreate(&gs,g,CU_STREAM_NON_BLOCKING,lo));
    int* out; CK(cudaMalloc(&out, 4096*4)); CK(cudaMemset(out,0xff,4096*4));
    void* a2[] = {&out, nullptr}; long spin=200000; a2[1]=&spin;
    cudaKernel_t k2; CK(cudaGetKernel(&k2,(const void*)smid_k));
    CD(cuLaunchKernel((CUfunction)k2,1024,1,1,128,1,1,0,gs,a2,nullptr));
    CD(cuStreamSynchronize(gs));
    std::vector<int> h(1024); CK(cudaMemcpy(h.data(),out,4096,cudaMemcpyDeviceToHost));
    std::set<int> sms(h.begin(),h.end()); printf("green want %u got part %u rem %u: kernel ran on %zu distinct SMs\n", want, part[0].sm.smCount, rem.sm.smCount, sms.size());
    // also runtime <<<>>> into green stream
    CK(cudaMemset(out,0xff,4096*4));
    smid_k<<<1024,128,0,(cudaStream_t)gs>>>(out, spin); cudaError_t e = cudaStreamSynchronize((cudaStream_t)gs);
    CK(cudaMemcpy(h.data(),out,4096,cudaMemcpyDeviceToHost));
    std::set<int> sms2(h.begin(),h.end()); printf("   runtime launch on green stream: err=%s SMs=%zu\n", cudaGetErrorString(e), sms2.size());
    // stream write on green stream
    CD(cuStreamWriteValue64(gs, dc, 777+want, 0)); CD(cuStreamSynchronize(gs)); printf("   green writeValue64 -> %llu\n", *(volatile unsigned long long*)hc);
    double a=now_us(); for(int i=0;i<N;i++) CD(cuLaunchKernel(f,1,1,1,32,1,1,0,gs,args,nullptr)); double b=now_us(); CD(cuStreamSynchronize(gs));
    printf("   green cuLaunchKernel(CUfunction primary): %.3f us\n",(b-a)/N);
    cudaFree(out);
  }
  printf("done\n");
  return 0;
}
