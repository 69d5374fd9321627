// alu_microbench.cu -- measured integer-pipe throughput of the instructions the evaluator
// issues (DPX VIMNMX / VIADDMNMX, IADD3, IMAD, ISETP+SEL) on this B200, to anchor the
// "alu" roofline.  Each kernel runs 8 independent dependency
// chains per thread on a full grid (8 CTAs x 256 threads per SM); rate = lane-ops / s.
// The PTX is asm volatile so NVVM cannot fold the chains; check the SASS mix with
//   cuobjdump -sass tools/alu_microbench
#include <cstdio>
#include <cuda_runtime.h>

#define CHAINS 8
#define ITERS 4096

template <int OP>
__global__ void __launch_bounds__(256) bench(int *out, int seed) {
    int a[CHAINS], b = seed ^ threadIdx.x, c = seed * 3 + blockIdx.x;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) a[i] = threadIdx.x * (i + 1) + seed;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int i = 0; i < CHAINS; ++i) {
            int x = a[i];
            if (OP == 0) {  // VIADDMNMX: max(x + b, c), then min(x + c, b)
                asm volatile("{.reg .s32 t; add.s32 t, %1, %2; max.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(b), "r"(c));
                asm volatile("{.reg .s32 t; add.s32 t, %1, %2; min.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(c), "r"(b));
            }
            if (OP == 1) {  // VIMNMX: max then min
                asm volatile("max.s32 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(b));
                asm volatile("min.s32 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(c));
            }
            if (OP == 2) {  // 3-input adds (IADD3)
                asm volatile("{.reg .s32 t; add.s32 t, %1, %2; add.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(b), "r"(c));
                asm volatile("{.reg .s32 t; sub.s32 t, %1, %2; add.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(c), "r"(b));
            }
            if (OP == 3) {  // IMAD
                asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(b), "r"(c));
                asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(c), "r"(b));
            }
            if (OP == 4) {  // ISETP + SEL
                asm volatile("{.reg .pred p; setp.gt.s32 p, %1, %2; selp.s32 %0, %1, %3, p;}" : "=r"(x) : "r"(x), "r"(c), "r"(b));
            }
            if (OP == 5) {  // IMAD + VIADDMNMX (one FMA-pipe, one ALU-pipe op)
                asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(b), "r"(c));
                asm volatile("{.reg .s32 t; add.s32 t, %1, %2; max.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(b), "r"(c));
            }
            if (OP == 6) {  // IMAD.HI (high word of a signed 32x32 product)
                asm volatile("mul.hi.s32 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(b));
                asm volatile("mad.hi.s32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(c), "r"(b));
            }
            if (OP == 7) {  // IMAD.HI + VIADDMNMX
                asm volatile("mul.hi.s32 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(b));
                asm volatile("{.reg .s32 t; add.s32 t, %1, %2; max.s32 %0, t, %3;}" : "=r"(x) : "r"(x), "r"(b), "r"(c));
            }
            if (OP == 8) {  // IMAD.IADD-style adds forced onto the FMA pipe: x * 1 + b
                asm volatile("mad.lo.s32 %0, %1, 1, %2;" : "=r"(x) : "r"(x), "r"(b));
                asm volatile("mad.lo.s32 %0, %1, 1, %2;" : "=r"(x) : "r"(x), "r"(c));
            }
            a[i] = x;
        }
        b += 1;
    }
    int s = 0;
#pragma unroll
    for (int i = 0; i < CHAINS; ++i) s += a[i];
    if (s == 0x7fffffff) out[0] = s;
}

template <int OP>
double run(const char *name, int ops_per_inner, int blocks, double clk_hz, int sms) {
    int *out;
    cudaMalloc(&out, 4);
    bench<OP><<<blocks, 256>>>(out, 1);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) bench<OP><<<blocks, 256>>>(out, r);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double lane_ops = 5.0 * blocks * 256.0 * ITERS * CHAINS * ops_per_inner;
    double rate = lane_ops / (ms / 1e3);
    double per_smsp_clk = rate / (sms * 4.0 * clk_hz);   // lane-ops per SMSP per clock (32 = 1 warp-instr/clk)
    printf("{\"op\": \"%s\", \"lane_ops_per_s\": %.4e, \"lanes_per_smsp_clk_at_max\": %.2f, \"ms\": %.3f}\n", name, rate,
           per_smsp_clk, ms);
    cudaFree(out);
    return rate;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const double hz = clk_khz * 1e3;
    const int sms = p.multiProcessorCount;
    const int blocks = sms * 8;
    printf("{\"sms\": %d, \"clock_mhz\": %.0f}\n", sms, hz / 1e6);
    run<0>("VIADDMNMX", 2, blocks, hz, sms);
    run<1>("VIMNMX", 2, blocks, hz, sms);
    run<2>("IADD3", 1, blocks, hz, sms);   // ptxas folds each pair into one IADD3
    run<3>("IMAD", 2, blocks, hz, sms);
    run<4>("ISETP+SEL", 2, blocks, hz, sms);
    run<5>("IMAD+VIADDMNMX", 2, blocks, hz, sms);
    run<6>("IMAD.HI", 2, blocks, hz, sms);
    run<7>("IMAD.HI+VIADDMNMX", 2, blocks, hz, sms);
    run<8>("IMAD.IADD(x*1+b)", 2, blocks, hz, sms);

    return 0;
}
