// Pipe-rate microbenchmark for the instruction mix of the sweep kernel (sm_100a).
// Each kernel runs N_ITER iterations of an unrolled block of independent ops
// (8 chains) and reports warp-instructions per cycle per SM.
#include <cstdio>
#include <cuda_runtime.h>

#define N_ITER 4096
#define CHAINS 8

__device__ __forceinline__ unsigned long long f2u(float a, float b) {
    unsigned long long r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r; }

template <int OP>
__global__ void k(float* out, float seed, long long* cyc)
{
    float v[2 * CHAINS];
    for (int c = 0; c < 2 * CHAINS; c++) v[c] = seed + threadIdx.x + c;
    int p[CHAINS];
    for (int c = 0; c < CHAINS; c++) p[c] = 0;
    const float a = seed * 0.5f, b = seed * 0.25f;
    long long t0 = clock64();
    for (int it = 0; it < N_ITER; it++) {
#pragma unroll
        for (int c = 0; c < CHAINS; c++) {
            if (OP == 0) {  // FFMA
                v[2 * c] = fmaf(v[2 * c], a, b);
            } else if (OP == 1) {  // FFMA2
                unsigned long long x = f2u(v[2 * c], v[2 * c + 1]), y = f2u(a, a), z = f2u(b, b), r;
                asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(x), "l"(y), "l"(z));
                asm("mov.b64 {%0,%1}, %2;" : "=f"(v[2 * c]), "=f"(v[2 * c + 1]) : "l"(r));
            } else if (OP == 2) {  // FADD2
                unsigned long long x = f2u(v[2 * c], v[2 * c + 1]), y = f2u(a, b), r;
                asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(x), "l"(y));
                asm("mov.b64 {%0,%1}, %2;" : "=f"(v[2 * c]), "=f"(v[2 * c + 1]) : "l"(r));
            } else if (OP == 3) {  // FSETP (OR-accumulate)
                int q = p[c];
                asm volatile("{.reg .pred t, u; setp.ne.u32 u, %0, 0; setp.le.or.f32 t, %1, %2, u; selp.u32 %0, 1, 0, t;}" : "+r"(q) : "f"(v[2 * c]), "f"(a));
                p[c] = q;
            } else if (OP == 4) {  // FMNMX3
                asm volatile("min.f32 %0, %0, %1;" : "+f"(v[2 * c]) : "f"(v[2 * c + 1]));
            } else if (OP == 5) {  // mix: 1 FFMA2 + 1 FSETP
                unsigned long long x = f2u(v[2 * c], v[2 * c + 1]), y = f2u(a, a), z = f2u(b, b), r;
                asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(x), "l"(y), "l"(z));
                asm("mov.b64 {%0,%1}, %2;" : "=f"(v[2 * c]), "=f"(v[2 * c + 1]) : "l"(r));
                int q = p[c];
                asm volatile("{.reg .pred t, u; setp.ne.u32 u, %0, 0; setp.le.or.f32 t, %1, %2, u; selp.u32 %0, 1, 0, t;}" : "+r"(q) : "f"(v[2 * c + 1]), "f"(b));
                p[c] = q;
            } else if (OP == 6) {  // FMUL (scalar)
                v[2 * c] = v[2 * c] * a;
            } else if (OP == 7) {  // IADD3
                int q = __float_as_int(v[2 * c]);
                asm volatile("add.s32 %0, %0, %1;" : "+r"(q) : "r"(__float_as_int(a)));
                v[2 * c] = __int_as_float(q);
            } else if (OP == 8) {  // MUFU.SQRT (sqrt.approx.ftz.f32): the XU pipe
                asm volatile("sqrt.approx.ftz.f32 %0, %0;" : "+f"(v[2 * c]));
            } else if (OP == 9) {  // MUFU.RSQ
                asm volatile("rsqrt.approx.ftz.f32 %0, %0;" : "+f"(v[2 * c]));
            } else if (OP == 10) {  // ISETP (OR-accumulate, signed compare of float bits)
                int q = p[c];
                asm volatile("{.reg .pred t, u; setp.ne.u32 u, %0, 0; setp.le.or.s32 t, %1, %2, u; selp.u32 %0, 1, 0, t;}"
                             : "+r"(q) : "r"(__float_as_int(v[2 * c])), "r"(__float_as_int(a)));
                p[c] = q;
            } else if (OP == 11) {  // FMNMX3 (3-input min)
                asm volatile("min.f32 %0, %0, %1, %2;" : "+f"(v[2 * c]) : "f"(v[2 * c + 1]), "f"(a));
            } else if (OP == 12) {  // F2I (cvt.rni.s32.f32), the conversion pipe
                int q;
                asm volatile("cvt.rni.s32.f32 %0, %1;" : "=r"(q) : "f"(v[2 * c]));
                v[2 * c] = __int_as_float(q) ;
            }
        }
    }
    long long t1 = clock64();
    float s = 0;
    for (int c = 0; c < 2 * CHAINS; c++) s += v[c];
    for (int c = 0; c < CHAINS; c++) s += p[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char* name, int warps_per_sm)
{
    int sms = 148, threads = 32 * warps_per_sm;
    float* out; long long* cyc;
    cudaMalloc(&out, sizeof(float) * sms * threads);
    cudaMalloc(&cyc, sizeof(long long) * sms);
    k<OP><<<sms, threads>>>(out, 1.0f, cyc);
    k<OP><<<sms, threads>>>(out, 1.0f, cyc);
    cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0; for (int i = 0; i < sms; i++) avg += h[i]; avg /= sms;
    double inst = (double)N_ITER * CHAINS * warps_per_sm * (OP == 5 ? 2 : 1);
    printf("%-8s warps/SM=%2d  warp-inst/clk/SM = %.3f  (lane-ops/clk/SM %.1f)\n", name, warps_per_sm, inst / avg,
           inst / avg * 32 * ((OP == 1 || OP == 2) ? 2 : 1));
    cudaFree(out); cudaFree(cyc);
}

int main()
{
    for (int w : {8, 16, 32}) {
        run<0>("FFMA", w); run<6>("FMUL", w); run<1>("FFMA2", w); run<2>("FADD2", w);
        run<3>("FSETP", w); run<4>("FMNMX", w); run<5>("FFMA2+SETP", w); run<7>("IADD", w);
        run<8>("MUFU.SQRT", w); run<9>("MUFU.RSQ", w); run<10>("ISETP", w); run<11>("FMNMX3", w); run<12>("F2I", w);
    }
    return 0;
}
