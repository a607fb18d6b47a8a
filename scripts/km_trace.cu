// Per-role timeline of the tensor-core k-means assignment (CTA 0, tiles 200..263): the kernel
// source compiled with -DKM_TRACE, lattice points as in config C4, k = 256.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DKM_TRACE -Ipaper_conf_icpp_komodamnm13_b200/csrc \
//      -Iinclude -o scripts/km_trace scripts/km_trace.cu
#include "../paper_conf_icpp_komodamnm13_b200/csrc/kmeans_tc.cu"

#include <cstdio>
#include <vector>

int main(int argc, char** argv) {
    const int k = 256, tiles_per_cta = 300;
    const int64_t n = (int64_t)148 * tiles_per_cta * 128;
    std::vector<float> x(n * 16);
    uint64_t st = 12345;
    auto rnd = [&]() { st = st * 6364136223846793005ull + 1442695040888963407ull; return (uint32_t)(st >> 33); };
    std::vector<float> cen(k * 16);
    for (int c = 0; c < k; ++c)
        for (int j = 0; j < 16; ++j) cen[c * 16 + j] = -64.f + 16.f * (float)(rnd() % 8);
    for (int64_t p = 0; p < n; ++p) {
        const int c = p < k ? (int)p : (int)(rnd() % k);
        for (int j = 0; j < 16; ++j) x[p * 16 + j] = cen[c * 16 + j] + (float)((int)(rnd() % 257) - 128) / 256.f;
    }
    for (int c = 0; c < k; ++c)
        for (int j = 0; j < 16; ++j) cen[c * 16 + j] = x[c * 16 + j];
    float *dx, *dc;
    int32_t* dm;
    int64_t *ds, *dn;
    int* de;
    cudaMalloc(&dx, n * 64);
    cudaMalloc(&dc, k * 64);
    cudaMalloc(&dm, n * 4);
    cudaMalloc(&ds, k * 16 * 8);
    cudaMalloc(&dn, k * 8);
    cudaMalloc(&de, 4);
    cudaMemcpy(dx, x.data(), n * 64, cudaMemcpyHostToDevice);
    cudaMemcpy(dc, cen.data(), k * 64, cudaMemcpyHostToDevice);
    float best = 1e30f;
    for (int rep = 0; rep < 8; ++rep) {
        cudaMemset(ds, 0, k * 16 * 8);
        cudaMemset(dn, 0, k * 8);
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        cudaEventRecord(a);
        cudaError_t e = accmg::k::kmeans_assign_tc(dx, dc, dm, ds, dn, 0, n, k, 8, de, 0, 148);
        cudaEventRecord(b);
        if (e != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
            printf("error %s\n", cudaGetErrorString(cudaGetLastError()));
            return 1;
        }
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep > 0 && ms < best) best = ms;
    }
    printf("# best of 7: %.4f ms for %lld points = %.1f cycles/tile at 1.965 GHz\n", best, (long long)n,
           best * 1.965e6 / tiles_per_cta);
#ifdef KM_TRACE
    unsigned long long tr[64][32];
    cudaMemcpyFromSymbol(tr, accmg::k::g_km_trace, sizeof(tr));
    for (int t = 0; t < 64; ++t) {
        printf("%d", t + 200);
        for (int ev = 0; ev < 32; ++ev) printf(" %lld", tr[t][ev] ? (long long)(tr[t][ev] - tr[0][9]) : -1ll);
        printf("\n");
    }
#endif
    return 0;
}
