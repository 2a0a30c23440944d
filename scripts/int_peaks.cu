// int_peaks.cu -- microbenchmark of the B200 integer pipes (SURVEY §8(d):
// "microbenchmark an IADD3/IMNMX/IMAD chain on the B200").  The roofline
// denominators of the scoring kernels (bench.py "roofline", bound "alu") come
// from the numbers this program prints, committed as MEASURED_INT_PEAKS.json.
//
// Each kernel runs NCH independent dependency chains per thread of one
// instruction kind (inline PTX, one SASS instruction per PTX op -- checked
// with cuobjdump -sass), 148 x BPS blocks of 256 threads, all resident at once.
// Per block, clock64() brackets the loop; lane-instructions per clock per SM =
// BPS x 256 x iters x ops_per_iter / mean block cycles.  CUDA events give the
// same count per second (the clock the SMs actually ran at is cycles / time).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/int_peaks scripts/int_peaks.cu
//   scripts/int_peaks            # one JSON object on stdout
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define NCH 8
#define UNR 8

enum { OP_IADD3 = 0, OP_IMNMX, OP_IMAD, OP_MIX_IADD3_IMAD, OP_IMAD_WIDE, OP_IADD64 };

template <int OP>
__device__ __forceinline__ void step(int (&x)[NCH], int y, int z) {
#pragma unroll
  for (int j = 0; j < NCH; j++) {
    if (OP == OP_IADD3) {  // x = x + y + z : IADD3
      asm volatile("{ add.s32 %0, %0, %1; }" : "+r"(x[j]) : "r"(y));
      asm volatile("{ add.s32 %0, %0, %1; }" : "+r"(x[j]) : "r"(z));
    } else if (OP == OP_IMNMX) {  // x = min(x, y); x = max(x, z) : 2 IMNMX
      asm volatile("{ min.s32 %0, %0, %1; }" : "+r"(x[j]) : "r"(y));
      asm volatile("{ max.s32 %0, %0, %1; }" : "+r"(x[j]) : "r"(z));
    } else if (OP == OP_IMAD) {  // x = x * y + z : IMAD
      asm volatile("{ mad.lo.s32 %0, %0, %1, %2; }" : "+r"(x[j]) : "r"(y), "r"(z));
    } else if (OP == OP_MIX_IADD3_IMAD) {  // even chains IADD3, odd chains IMAD
      if (j & 1) asm volatile("{ mad.lo.s32 %0, %0, %1, %2; }" : "+r"(x[j]) : "r"(y), "r"(z));
      else asm volatile("{ add.s32 %0, %0, %1; }" : "+r"(x[j]) : "r"(y));
    }
  }
}

template <int OP>
__global__ void __launch_bounds__(256) k_int(int iters, int y, int z, int *sink, long long *cyc) {
  int x[NCH];
#pragma unroll
  for (int j = 0; j < NCH; j++) x[j] = threadIdx.x + j;
  __syncthreads();
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int u = 0; u < UNR; u++) step<OP>(x, y, z);
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int j = 0; j < NCH; j++) acc ^= x[j];
  if (acc == 0x7fffffff) sink[0] = acc;
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// 64-bit multiply-add / add chains (accsum accumulation in the scoring kernels)
template <int OP>
__global__ void __launch_bounds__(256) k_int64(int iters, int y, long long z, long long *sink, long long *cyc) {
  long long x[NCH];
#pragma unroll
  for (int j = 0; j < NCH; j++) x[j] = threadIdx.x + j;
  __syncthreads();
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int u = 0; u < UNR; u++) {
#pragma unroll
      for (int j = 0; j < NCH; j++) {
        if (OP == OP_IMAD_WIDE)  // x += lo32(x) * y : IMAD.WIDE (the product depends on the chain)
          asm volatile("{ .reg .s32 lo; cvt.u32.u64 lo, %0; mad.wide.s32 %0, lo, %1, %0; }" : "+l"(x[j]) : "r"(y));
        else  // x += z (64-bit add)
          asm volatile("{ add.s64 %0, %0, %1; }" : "+l"(x[j]) : "l"(z));
      }
    }
  }
  long long t1 = clock64();
  long long acc = 0;
#pragma unroll
  for (int j = 0; j < NCH; j++) acc ^= x[j];
  if (acc == 0x7fffffffffffll) sink[0] = acc;
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

struct Res {
  double lanes_per_clk_sm, lane_ops_per_s, mhz_eff;
};

template <class F>
static Res run(F launch, int blocks, int threads, long long ops_per_thread, long long *d_cyc) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  launch();  // warm-up
  cudaDeviceSynchronize();
  float best = 1e30f;
  std::vector<long long> cyc(blocks);
  double best_cyc = 0;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(a);
    launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) {
      best = ms;
      cudaMemcpy(cyc.data(), d_cyc, blocks * 8, cudaMemcpyDeviceToHost);
      double s = 0;
      for (long long c : cyc) s += (double)c;
      best_cyc = s / blocks;
    }
  }
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const double bps = (double)blocks / sms;
  Res r;
  r.lanes_per_clk_sm = bps * threads * (double)ops_per_thread / best_cyc;
  r.lane_ops_per_s = (double)blocks * threads * (double)ops_per_thread / (best * 1e-3);
  r.mhz_eff = best_cyc / (best * 1e-3) / 1e6;
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  return r;
}

int main(int argc, char **argv) {
  int sms = 0, clk_khz = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  const int BPS = 4, threads = 256, blocks = sms * BPS;
  const int iters = argc > 1 ? atoi(argv[1]) : 32768;
  int *sink;
  long long *sink64, *cyc;
  cudaMalloc(&sink, 64);
  cudaMalloc(&sink64, 64);
  cudaMalloc(&cyc, blocks * 8);
  const long long per32 = (long long)iters * UNR * NCH;
  struct Item {
    const char *name, *pipe, *sass;
    long long ops;
    Res r;
  } items[8];
  int n = 0;
#define RUN32(OP, NAME, PIPE, SASS, OPS)                                                                   \
  items[n].name = NAME; items[n].pipe = PIPE; items[n].sass = SASS; items[n].ops = OPS;                  \
  items[n].r = run([&] { k_int<OP><<<blocks, threads>>>(iters, 3, 5, sink, cyc); }, blocks, threads, OPS, cyc); n++;
  // counts are SASS instructions per thread (ptxas merges the two add.s32 into one IADD3)
  RUN32(OP_IADD3, "add.s32 + add.s32 (one IADD3)", "alu", "IADD3", per32);
  RUN32(OP_IMNMX, "min.s32, max.s32 (two VIMNMX)", "alu", "VIMNMX", per32 * 2);
  RUN32(OP_IMAD, "mad.lo.s32 (IMAD)", "fma", "IMAD", per32);
  RUN32(OP_MIX_IADD3_IMAD, "add.s32 || mad.lo.s32 on alternate chains (IADD3 || IMAD, 1:1)", "alu+fma",
        "IADD3,IMAD", per32);
#define RUN64(OP, NAME, PIPE, SASS, OPS)                                                                   \
  items[n].name = NAME; items[n].pipe = PIPE; items[n].sass = SASS; items[n].ops = OPS;                  \
  items[n].r = run([&] { k_int64<OP><<<blocks, threads>>>(iters, 3, 5, sink64, cyc); }, blocks, threads, OPS, cyc); n++;
  RUN64(OP_IMAD_WIDE, "mad.wide.s32 as ptxas emits it (IMAD.WIDE + IADD3 + IADD3.X per op; counted as 1 op)", "fma+alu", "IMAD.WIDE,IADD3,IADD3.X", per32);
  RUN64(OP_IADD64, "add.s64 (IADD3 + IADD3.X)", "alu", "IADD3,IADD3.X", per32 * 2);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    fprintf(stderr, "CUDA error: %s\n", cudaGetErrorString(e));
    return 1;
  }
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, 0);
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"attr_clock_mhz\": %.0f, \"blocks_per_sm\": %d, \"threads\": %d, "
         "\"chains_per_thread\": %d, \"how\": \"scripts/int_peaks.cu: NCH independent chains per thread of one PTX op, "
         "clock64 per block (lanes/clk/SM), CUDA events best of 5 (lane-ops/s)\", \"ops\": [",
         prop.name, sms, clk_khz / 1e3, BPS, threads, NCH);
  for (int i = 0; i < n; i++)
    printf("%s{\"op\": \"%s\", \"pipe\": \"%s\", \"sass\": \"%s\", \"lane_ops_per_clk_per_sm\": %.2f, "
           "\"lane_ops_per_s\": %.4e, \"effective_mhz\": %.0f}",
           i ? ", " : "", items[i].name, items[i].pipe, items[i].sass, items[i].r.lanes_per_clk_sm,
           items[i].r.lane_ops_per_s, items[i].r.mhz_eff);
  printf("]}\n");
  return 0;
}
