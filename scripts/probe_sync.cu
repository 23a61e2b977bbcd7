// probe_sync.cu -- barrier costs on this GPU (diagnostic, not part of liblf.so):
//   grid.sync() of a cooperative launch at several grid sizes, cluster.sync() at cluster
//   sizes 8 / 16, and whether a cooperative launch may also carry a cluster dimension.
// build+run: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/probe_sync scripts/probe_sync.cu && /tmp/probe_sync
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>

namespace cg = cooperative_groups;

__global__ void k_grid(int iters, int* sink) {
    cg::grid_group g = cg::this_grid();
    int x = 0;
    for (int i = 0; i < iters; i++) {
        x += sink[(blockIdx.x + i) & 63];
        g.sync();
    }
    if (x == 12345) sink[0] = x;
}

__global__ void k_cluster(int iters, int* sink) {
    cg::cluster_group c = cg::this_cluster();
    int x = 0;
    for (int i = 0; i < iters; i++) {
        x += sink[(blockIdx.x + i) & 63];
        c.sync();
    }
    if (x == 12345) sink[0] = x;
}

// cooperative + cluster: grid barrier first, then cluster barriers in cluster 0 only
__global__ void k_both(int iters, int* sink) {
    cg::grid_group g = cg::this_grid();
    cg::cluster_group c = cg::this_cluster();
    int x = 0;
    for (int i = 0; i < 4; i++) {
        x += sink[(blockIdx.x + i) & 63];
        g.sync();
    }
    if (blockIdx.x >= c.num_blocks()) return;
    for (int i = 0; i < iters; i++) {
        x += sink[(blockIdx.x + i) & 63];
        c.sync();
    }
    if (x == 12345) sink[0] = x;
}

static float time_it(cudaLaunchConfig_t& cfg, void (*k)(int, int*), int iters, int* sink) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaError_t e = cudaLaunchKernelEx(&cfg, k, iters, sink);  // warm-up
    if (e != cudaSuccess) { printf("  launch error: %s\n", cudaGetErrorString(e)); cudaGetLastError(); return -1; }
    cudaDeviceSynchronize();
    cudaEventRecord(a, cfg.stream);
    cudaLaunchKernelEx(&cfg, k, iters, sink);
    cudaEventRecord(b, cfg.stream);
    e = cudaEventSynchronize(b);
    if (e != cudaSuccess) { printf("  run error: %s\n", cudaGetErrorString(e)); return -1; }
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
}

int main() {
    int* sink;
    cudaMalloc(&sink, 4096);
    cudaMemset(sink, 0, 4096);
    const int iters = 1000;
    cudaLaunchAttribute at[2];
    cudaLaunchConfig_t cfg = {};
    cfg.stream = 0;
    cfg.attrs = at;
    for (int threads : {512, 1024}) {
        for (int grid : {16, 32, 74, 148}) {
            cfg.gridDim = dim3(grid);
            cfg.blockDim = dim3(threads);
            at[0].id = cudaLaunchAttributeCooperative;
            at[0].val.cooperative = 1;
            cfg.numAttrs = 1;
            const float t0 = time_it(cfg, k_grid, 1, sink);
            const float t = time_it(cfg, k_grid, iters, sink);
            printf("grid.sync   grid=%3d threads=%4d: %.3f us per barrier\n", grid, threads, (t - t0) * 1e3f / (iters - 1));
        }
    }
    cudaFuncSetAttribute((const void*)k_cluster, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaFuncSetAttribute((const void*)k_both, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    for (int threads : {512, 1024}) {
        for (int cs : {4, 8, 16}) {
            cfg.gridDim = dim3(cs);
            cfg.blockDim = dim3(threads);
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = cs;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            cfg.numAttrs = 1;
            const float t0 = time_it(cfg, k_cluster, 1, sink);
            const float t = time_it(cfg, k_cluster, iters, sink);
            printf("cluster.sync cs=%2d threads=%4d: %.3f us per barrier\n", cs, threads, (t - t0) * 1e3f / (iters - 1));
        }
    }
    for (int cs : {8, 16}) {
        int grid = (148 / cs) * cs;
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(512);
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = cs;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        at[1].id = cudaLaunchAttributeCooperative;
        at[1].val.cooperative = 1;
        cfg.numAttrs = 2;
        int maxc = 0;
        cudaOccupancyMaxActiveClusters(&maxc, (const void*)k_both, &cfg);
        printf("coop+cluster cs=%d: max active clusters %d\n", cs, maxc);
        for (int g2 : {grid, maxc * cs}) {
            if (g2 <= 0) continue;
            cfg.gridDim = dim3(g2);
            const float t0 = time_it(cfg, k_both, 1, sink);
            const float t = time_it(cfg, k_both, iters, sink);
            printf("coop+cluster cs=%2d grid=%3d: %s %.3f us per cluster barrier\n", cs, g2, t0 < 0 ? "FAILED" : "ok",
                   (t - t0) * 1e3f / (iters - 1));
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("final: %s\n", cudaGetErrorString(e));
    return 0;
}
