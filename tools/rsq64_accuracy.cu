// Dev probe: accuracy of rsqrt.approx.ftz.f64 (MUFU.RSQ64H) vs exact 1/sqrt in double.
#include <cstdio>
#include <cmath>
#include <cuda_runtime.h>
__global__ void k(const double* x, double* y, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) { double r; asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x[i])); y[i] = r; }
}
int main() {
    const int n = 1 << 20;
    double *hx = new double[n], *hy = new double[n];
    for (int i = 0; i < n; ++i) hx[i] = 1e-4 + 12.0 * ((i * 2654435761u) % 1000003) / 1000003.0;
    double *dx, *dy;
    cudaMalloc(&dx, n * 8); cudaMalloc(&dy, n * 8);
    cudaMemcpy(dx, hx, n * 8, cudaMemcpyHostToDevice);
    k<<<n / 256, 256>>>(dx, dy, n);
    cudaMemcpy(hy, dy, n * 8, cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int i = 0; i < n; ++i) { double e = fabs(hy[i] * sqrt(hx[i]) - 1.0); if (e > mx) mx = e; }
    printf("{\"what\": \"rsqrt.approx.ftz.f64 max rel err\", \"value\": %.3e, \"log2\": %.2f}\n", mx, log2(mx));
    return 0;
}
