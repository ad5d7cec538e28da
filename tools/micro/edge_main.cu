// Standalone driver for K1 (bisecting): includes edge.cu, launches one 256x256 image.
#include "../../paper_conf_ipps_sundaramrc09_b200/csrc/kernels/edge.cu"
#include <cstdio>
#include <vector>
int main() {
    const int H = 256, W = 256;
    float *in, *out;
    cudaMalloc(&in, H * W * 4); cudaMalloc(&out, H * W * 4);
    std::vector<float> h(H * W);
    for (int i = 0; i < H * W; ++i) h[i] = (i * 37 % 255) / 255.f;
    cudaMemcpy(in, h.data(), H * W * 4, cudaMemcpyHostToDevice);
    std::vector<float> k1(256), k2(256);
    for (int i = 0; i < 256; ++i) { k1[i] = (i % 7) * 0.01f; k2[i] = (i % 5) * -0.01f; }
    tg::EdgeArgs a{};
    a.in = in; a.in_img_stride = H * W; a.in_row0 = 0; a.in_rows = H;
    a.out = out; a.out_img_stride = H * W; a.out_row0 = 0; a.out_rows = H; a.H = H; a.W = W; a.nimg = 1;
    a.k1_host = k1.data(); a.k2_host = k2.data(); a.ks = 16;
    cudaError_t e = tg::launch_edge(a, 0);
    printf("launch: %s\n", cudaGetErrorString(e));
    printf("sync: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    std::vector<float> o(H * W);
    cudaMemcpy(o.data(), out, H * W * 4, cudaMemcpyDeviceToHost);
    double s = 0; for (float v : o) s += v;
    printf("checksum %.6f\n", s);
    return 0;
}
