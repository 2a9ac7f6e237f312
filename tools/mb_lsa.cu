// Dev feasibility check: NCCL 2.28 symmetric window on a one-rank communicator;
// LSA pointer of the (self) peer computed on the device, written through.
//   nvcc -gencode arch=compute_100a,code=sm_100a -std=c++17 -I$NCCL/include tools/mb_lsa.cu -L$NCCL/lib -l:libnccl.so.2 -Xlinker -rpath,$NCCL/lib -o tools/mb_lsa
#include <cstdio>
#include <nccl.h>
#include <nccl_device.h>
__global__ void k_ptr(ncclWindow_t w, int peer, void **out) { out[0] = ncclGetLsaPointer(w, 0, peer); }
__global__ void k_write(int *p, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) p[i] = 3 * i + 1;
}
#define CK(x) do { auto r = (x); if ((int)r) { printf("%s failed: %d line %d\n", #x, (int)r, __LINE__); return 1; } } while (0)
int main() {
  ncclComm_t comm; int dev = 0;
  CK(ncclCommInitAll(&comm, 1, &dev));
  void *buf; size_t bytes = 1 << 22;
  CK(ncclMemAlloc(&buf, bytes));
  ncclWindow_t win;
  CK(ncclCommWindowRegister(comm, buf, bytes, &win, NCCL_WIN_COLL_SYMMETRIC));
  ncclDevComm dcomm; ncclDevCommRequirements req = {};
  req.lsaBarrierCount = 1;
  ncclResult_t r = ncclDevCommCreate(comm, &req, &dcomm);
  printf("ncclDevCommCreate -> %d\n", (int)r);
  void **d_out; cudaMalloc(&d_out, 8);
  k_ptr<<<1, 1>>>(win, 0, d_out);
  void *lsa = nullptr; cudaMemcpy(&lsa, d_out, 8, cudaMemcpyDeviceToHost);
  printf("local %p lsa(self) %p  err=%s\n", buf, lsa, cudaGetErrorString(cudaGetLastError()));
  const int n = 1 << 20;
  k_write<<<64, 256>>>((int *)lsa, n);
  cudaDeviceSynchronize();
  int h[4]; cudaMemcpy(h, (int *)buf + 1000, 16, cudaMemcpyDeviceToHost);
  printf("through lsa pointer: %d %d %d %d (expect 3001 3004 3007 3010) err=%s\n", h[0], h[1], h[2], h[3],
         cudaGetErrorString(cudaGetLastError()));
  ncclCommWindowDeregister(comm, win);
  ncclMemFree(buf);
  ncclCommDestroy(comm);
  return 0;
}
