// Self-test of groupby.cu's hand-written radix sort and scans on random keys
// (built and run on the GPU box by hand when debugging: nvcc -arch=sm_100a).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <string>
#include <mutex>
#include "../include/up.h"
up_status up_internal_fail(up_status st, const std::string &) { return st; }
void up_internal_add_launches(up_ctx *, long long) {}
up_status up_internal_scratch(up_ctx *, size_t, void **) { return UP_OK; }
static std::mutex g_mu;
extern "C" int32_t up_limbs(int32_t) { return 1; }
std::mutex &up_internal_mutex(up_ctx *) { return g_mu; }
#include "../paper_conf_icde_lixylz24_b200/csrc/groupby.cu"

int main() {
    for (long long n : {1ll, 100ll, 4096ll, 5000ll, 100000ll, 3000001ll}) {
        std::vector<uint32_t> hk(n), hv(n);
        srand(7);
        for (long long i = 0; i < n; ++i) { hk[i] = (uint32_t)rand() * 2654435761u; hv[i] = (uint32_t)i; }
        uint32_t *k, *v, *k2, *v2, *cnt, *part;
        const long long nt = (n + RS_TILE - 1) / RS_TILE;
        cudaMalloc(&k, 4 * n); cudaMalloc(&v, 4 * n); cudaMalloc(&k2, 4 * n); cudaMalloc(&v2, 4 * n);
        cudaMalloc(&cnt, 4 * (RADIX * nt + 64)); cudaMalloc(&part, 4 * ((RADIX * nt > n ? RADIX * nt : n) / SCAN_CHUNK + 64));
        cudaMemcpy(k, hk.data(), 4 * n, cudaMemcpyHostToDevice);
        cudaMemcpy(v, hv.data(), 4 * n, cudaMemcpyHostToDevice);
        long long launches = 0;
        {   // stage check: histogram + scan of the first digit pass against the host
            const int grid = (int)(nt < 148 * 8 ? nt : 148 * 8);
            k_rs_hist<<<grid, RS_THREADS>>>(k, n, 0, cnt, nt);
            std::vector<uint32_t> hc(RADIX * nt), want(RADIX * nt, 0);
            cudaMemcpy(hc.data(), cnt, 4 * RADIX * nt, cudaMemcpyDeviceToHost);
            for (long long i = 0; i < n; ++i) want[(hk[i] & 255u) * nt + i / RS_TILE]++;
            long long hbad = 0;
            for (long long i = 0; i < RADIX * nt; ++i) hbad += hc[i] != want[i];
            {
                const long long m = (long long)RADIX * nt, nc = (m + SCAN_CHUNK - 1) / SCAN_CHUNK;
                k_scan_sums<<<(unsigned)nc, 256>>>(cnt, m, part);
                uint32_t p0 = 0; cudaMemcpy(&p0, part, 4, cudaMemcpyDeviceToHost);
                k_scan_parts<<<1, 1024>>>(part, nc);
                uint32_t p1 = 0; cudaMemcpy(&p1, part, 4, cudaMemcpyDeviceToHost);
                k_scan_apply<<<(unsigned)nc, 256>>>(cnt, cnt, m, part, 0);
                printf("  part after sums %u after parts %u (%s)\n", p0, p1, cudaGetErrorString(cudaDeviceSynchronize()));
            }
            cudaMemcpy(hc.data(), cnt, 4 * RADIX * nt, cudaMemcpyDeviceToHost);
            uint32_t acc = 0; long long sbad = 0;
            for (long long i = 0; i < RADIX * nt; ++i) { sbad += hc[i] != acc; acc += want[i]; }
            printf("n=%lld hist bad=%lld scan bad=%lld (%s) first offsets %u %u %u\n", n, hbad, sbad,
                   cudaGetErrorString(cudaDeviceSynchronize()), hc[0], hc[nt], hc[2 * nt]);
        }
        cudaError_t e = radix_sort_pairs(k, v, k2, v2, n, 32, cnt, part, 0, launches);
        cudaError_t e2 = cudaDeviceSynchronize();
        std::vector<uint32_t> ok(n), ov(n);
        cudaMemcpy(ok.data(), k, 4 * n, cudaMemcpyDeviceToHost);
        cudaMemcpy(ov.data(), v, 4 * n, cudaMemcpyDeviceToHost);
        std::vector<uint32_t> order(n);
        for (long long i = 0; i < n; ++i) order[i] = (uint32_t)i;
        std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return hk[a] < hk[b]; });
        long long bad = 0;
        for (long long i = 0; i < n; ++i) bad += (ov[i] != order[i]) || (ok[i] != hk[order[i]]);
        // scan check
        std::vector<uint32_t> hs(n);
        for (long long i = 0; i < n; ++i) hs[i] = (uint32_t)(i % 3 == 0);
        cudaMemcpy(k2, hs.data(), 4 * n, cudaMemcpyHostToDevice);
        scan_u32(k2, v2, n, part, true, 0, launches);
        cudaDeviceSynchronize();
        std::vector<uint32_t> so(n);
        cudaMemcpy(so.data(), v2, 4 * n, cudaMemcpyDeviceToHost);
        long long sbad = 0; uint32_t acc = 0;
        for (long long i = 0; i < n; ++i) { acc += hs[i]; sbad += so[i] != acc; }
        printf("n=%lld sort %s/%s bad=%lld scan bad=%lld\n", n, cudaGetErrorString(e), cudaGetErrorString(e2), bad, sbad);
        cudaFree(k); cudaFree(v); cudaFree(k2); cudaFree(v2); cudaFree(cnt); cudaFree(part);
    }
    return 0;
}
