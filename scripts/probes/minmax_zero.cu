// Probe: bit patterns of max/min (plain, .NaN) on +-0 and NaN inputs on this GPU (R12 evidence).
#include <cstdio>
#include <cstdint>
#include <cstring>
__global__ void k(const float *in, uint32_t *out) {
    float a = in[0], b = in[1], n = in[2];
    float r[8];
    asm("max.f32 %0, %1, %2;" : "=f"(r[0]) : "f"(a), "f"(b));
    asm("max.f32 %0, %1, %2;" : "=f"(r[1]) : "f"(b), "f"(a));
    asm("min.f32 %0, %1, %2;" : "=f"(r[2]) : "f"(a), "f"(b));
    asm("min.f32 %0, %1, %2;" : "=f"(r[3]) : "f"(b), "f"(a));
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r[4]) : "f"(a), "f"(b));
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r[5]) : "f"(b), "f"(a));
    asm("min.NaN.f32 %0, %1, %2;" : "=f"(r[6]) : "f"(a), "f"(b));
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r[7]) : "f"(n), "f"(a));
    for (int i = 0; i < 8; ++i) out[i] = __float_as_uint(r[i]);
}
int main() {
    uint32_t nb = 0x7fc01234u; float nanv; memcpy(&nanv, &nb, 4);
    float h[3] = {-0.0f, 0.0f, nanv};
    float *d; uint32_t *o; uint32_t ho[8];
    cudaMalloc(&d, 12); cudaMalloc(&o, 32);
    cudaMemcpy(d, h, 12, cudaMemcpyHostToDevice);
    k<<<1, 1>>>(d, o);
    cudaMemcpy(ho, o, 32, cudaMemcpyDeviceToHost);
    const char *nm[8] = {"max(-0,+0)", "max(+0,-0)", "min(-0,+0)", "min(+0,-0)", "max.NaN(-0,+0)",
                         "max.NaN(+0,-0)", "min.NaN(-0,+0)", "max.NaN(NaN(0x7fc01234),-0)"};
    for (int i = 0; i < 8; ++i) printf("%-30s 0x%08x\n", nm[i], ho[i]);
    return 0;
}
