// repro_vimnmx3.cu -- ptxas (CUDA 12.9, sm_100a) folds an operand negation into VIMNMX3
// and loses it: -min(min(a, -(x + y)), c) computes with +(x + y).  Found by the GPU
// parity tests (evaluator cost != exact re-evaluation).  Each kernel below is one
// pattern; main() prints ok / MISMATCH per pattern.  See DESIGN.md "Compiler erratum".
#include <algorithm>
#include <cstdio>

__global__ void k(const int *in, int *out) {
    const int t = threadIdx.x;
    int i0 = in[t * 3 + 0], i1 = in[t * 3 + 1], i2 = in[t * 3 + 2];
    int nf0 = -i0, nf1 = -i1 + nf0, nf2 = -i2;
    out[t * 8 + 0] = -min(min(nf0, nf1), nf2);          // 3-input min, negated operands
    out[t * 8 + 1] = -min(nf0, nf1);                    // 2-input min, negated operand
    out[t * 8 + 2] = __viaddmax_s32(nf1, i2, nf0);      // add+max with negated operand
    out[t * 8 + 3] = min(min(i0, i1 + i0), i2);         // 3-input min, no negation
    out[t * 8 + 4] = max(max(nf0, nf1), nf2);           // 3-input max, negated operands
    out[t * 8 + 5] = min(min(nf0, nf1), nf2);           // 3-input min, negated operands, no outer neg
    out[t * 8 + 6] = nf1;
    out[t * 8 + 7] = 0;
}

int main() {
    const int n = 4;
    int h[3 * n] = {6, 3448, 619, 1, 2, 3, 100, 5, 7, 0, 0, 9};
    int *d, *o;
    cudaMalloc(&d, sizeof h);
    cudaMalloc(&o, 8 * n * 4);
    cudaMemcpy(d, h, sizeof h, cudaMemcpyHostToDevice);
    k<<<1, n>>>(d, o);
    int r[8 * n];
    cudaMemcpy(r, o, sizeof r, cudaMemcpyDeviceToHost);
    const char *names[] = {"-min3(neg)", "-min2(neg)", "viaddmax(neg)", "min3(plain)", "max3(neg)", "min3(neg)"};
    int bad = 0;
    for (int t = 0; t < n; ++t) {
        long i0 = h[3 * t], i1 = h[3 * t + 1], i2 = h[3 * t + 2];
        long nf0 = -i0, nf1 = -i1 + nf0, nf2 = -i2;
        long want[6] = {-std::min(std::min(nf0, nf1), nf2), -std::min(nf0, nf1), std::max(nf1 + i2, nf0),
                        std::min(std::min(i0, i1 + i0), i2), std::max(std::max(nf0, nf1), nf2),
                        std::min(std::min(nf0, nf1), nf2)};
        for (int c = 0; c < 6; ++c)
            if (r[8 * t + c] != want[c]) {
                printf("MISMATCH t%d %s gpu %d want %ld\n", t, names[c], r[8 * t + c], want[c]);
                ++bad;
            }
    }
    printf("%s (%d mismatches)\n", bad ? "BUG REPRODUCED" : "all ok", bad);
    return 0;
}
