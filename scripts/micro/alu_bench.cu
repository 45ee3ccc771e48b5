// Throughput of the epilogue's integer instructions on sm_100a: cycles per warp instruction per
// SMSP for IMAD.HI (64-bit addend), SHF.R.S32.HI, I2IP.U4.S32.SAT, IMAD, IADD3, LOP3, PRMT,
// FFMA, F2I, I2F (8 independent chains per thread, 4..16 warps per SM).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

template <int OP>
__global__ void alu(int iters, long long *out, int *sink, int a0, int b0) {
    int x[8];
    int64_t c = (static_cast<int64_t>(b0) << 33) + a0;
#pragma unroll
    for (int j = 0; j < 8; ++j) x[j] = threadIdx.x * 7 + j * 13 + a0;
    float f[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) f[j] = static_cast<float>(x[j]);
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            if (OP == 0) asm volatile("{\n\t.reg .s64 t;\n\tmul.wide.s32 t, %0, %1;\n\tadd.s64 t, t, %2;\n\tshr.s64 t, t, 32;\n\tcvt.u32.u64 %0, t;\n\t}" : "+r"(x[j]) : "r"(b0), "l"(c));   // IMAD.HI
            if (OP == 1) { int r; asm volatile("shf.r.clamp.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(x[j]), "r"(x[j]), "r"(b0)); x[j] = r; }
            if (OP == 2) { int r; asm volatile("cvt.pack.sat.u4.s32.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(x[j]), "r"(a0), "r"(x[j])); x[j] = r; }
            if (OP == 3) x[j] = x[j] * b0 + a0;                                                          // IMAD
            if (OP == 4) { asm volatile("add.s32 %0, %0, %1;" : "+r"(x[j]) : "r"(b0)); }                 // IADD
            if (OP == 5) { asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x[j]) : "r"(b0), "r"(a0)); }
            if (OP == 6) { asm volatile("prmt.b32 %0, %0, %1, 0x3210;" : "+r"(x[j]) : "r"(b0)); }
            if (OP == 7) f[j] = __fmaf_rn(f[j], 1.0001f, 0.5f);
            if (OP == 8) { asm volatile("shr.s32 %0, %0, %1;" : "+r"(x[j]) : "r"(b0)); }
            if (OP == 10) { asm volatile("mad.hi.s32 %0, %0, %1, %2;" : "+r"(x[j]) : "r"(b0), "r"(a0)); }
            if (OP == 11) { asm volatile("mul.hi.u32 %0, %0, %1;" : "+r"(x[j]) : "r"(b0)); }
            if (OP == 12) { asm volatile("{\n\t.reg .s64 t;\n\tmul.wide.s32 t, %0, %1;\n\tcvt.u32.u64 %0, t;\n\t}" : "+r"(x[j]) : "r"(b0)); }
            if (OP == 13) { asm volatile("{\n\t.reg .s64 t;\n\tmad.wide.s32 t, %0, %1, %2;\n\tmov.b64 {%0, _}, t;\n\t}" : "+r"(x[j]) : "r"(b0), "l"(c)); }
            if (OP == 14) { float r; asm volatile("cvt.rn.f32.s32 %0, %1;" : "=f"(r) : "r"(x[j])); f[j] += r; }
            if (OP == 15) { int r; asm volatile("cvt.rmi.s32.f32 %0, %1;" : "=r"(r) : "f"(f[j])); x[j] += r; f[j] += 1.0f; }
            if (OP == 16) { asm volatile("{\n\t.reg .s64 t;\n\tmul.wide.s32 t, %0, %1;\n\tadd.s64 t, t, %2;\n\tshr.s64 t, t, 40;\n\tcvt.u32.u64 %0, t;\n\t}" : "+r"(x[j]) : "r"(b0), "l"(c)); }
            if (OP == 17) { double d = __longlong_as_double((static_cast<long long>(0x43300000) << 32) | static_cast<unsigned>(x[j]));
                            d = __fma_rn(d, 1.0000001, -4503599627370496.0); x[j] = static_cast<int>(__double_as_longlong(d)); }
            if (OP == 18) { double d = __longlong_as_double((static_cast<long long>(0x43300000) << 32) | static_cast<unsigned>(x[j]));
                            d = __dadd_rd(d, 1.5); x[j] = static_cast<int>(__double_as_longlong(d)); }
            if (OP == 19) { double d; asm volatile("cvt.rn.f64.s32 %0, %1;" : "=d"(d) : "r"(x[j])); x[j] = static_cast<int>(__double_as_longlong(d) >> 20); }
            if (OP == 9) { int r; asm volatile("min.s32 %0, %1, %2;" : "=r"(r) : "r"(x[j]), "r"(b0)); x[j] = r + 1; }
        }
    }
    long long t1 = clock64();
    int s = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) s += x[j] + static_cast<int>(f[j]);
    if (s == 0x7fff1234) sink[0] = s;
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

int main() {
    long long *out; cudaMalloc(&out, 148 * 8);
    int *sink; cudaMalloc(&sink, 64);
    const char *names[] = {"IMAD.HI(+64b)", "SHF(funnel)", "I2IP.U4.SAT", "IMAD", "IADD", "LOP3", "PRMT", "FFMA", "SHR.S32", "IMNMX+IADD", "mad.hi.s32", "mul.hi.u32", "mul.wide.lo", "mad.wide", "I2F+FADD", "F2I.floor+..", "wide>>40", "DFMA", "DADD.RD", "I2F.F64"};
    for (int op = 0; op < 20; ++op)
        for (int warps : {4, 8, 16}) {
            const int iters = 2048;
            for (int rep = 0; rep < 2; ++rep) {
                switch (op) {
                case 0: alu<0><<<148, warps * 32>>>(iters, out, sink, 3, 1 << 30); break;
                case 1: alu<1><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 2: alu<2><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 3: alu<3><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 4: alu<4><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 5: alu<5><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 6: alu<6><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 7: alu<7><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 8: alu<8><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 9: alu<9><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 10: alu<10><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 11: alu<11><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 12: alu<12><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 13: alu<13><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 14: alu<14><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 15: alu<15><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 16: alu<16><<<148, warps * 32>>>(iters, out, sink, 3, 1 << 30); break;
                case 17: alu<17><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 18: alu<18><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                case 19: alu<19><<<148, warps * 32>>>(iters, out, sink, 3, 5); break;
                }
            }
            cudaDeviceSynchronize();
            long long h; cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
            const double ins = static_cast<double>(warps) * iters * 32 / 4;   // warp instructions per SMSP
            printf("%-14s warps=%2d  cycles/warp-instr/SMSP = %.2f\n", names[op], warps, h / ins);
        }
    return 0;
}
