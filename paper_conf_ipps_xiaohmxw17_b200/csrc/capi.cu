// Host-side bookkeeping of the C ABI: status strings, CUDA error capture,
// launch counting, device properties.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <atomic>
#include <cstdio>
#include <cstring>

#include "dda_internal.cuh"

namespace dda {
namespace {
std::atomic<int64_t> g_launches{0};
thread_local char g_last_err[256] = "";
}  // namespace

void note_launch(int k) { g_launches.fetch_add(k, std::memory_order_relaxed); }

dda_status_t cuda_fail(cudaError_t e) {
    std::snprintf(g_last_err, sizeof g_last_err, "%s: %s", cudaGetErrorName(e), cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? DDA_ERR_OOM : DDA_ERR_CUDA;
}

int device_sms() {
    static int cached_dev = -1, cached = 148;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev != cached_dev) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0) cached = v;
        cached_dev = dev;
    }
    return cached;
}

void trace(const char* what) {
    static int on = -1;
    if (on < 0) {
        const char* e = getenv("DDA_TRACE");
        on = (e && e[0] == '1') ? 1 : 0;
    }
    if (!on) return;
    static auto last = std::chrono::steady_clock::now();
    const auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "[dda trace] %-28s +%9.1f us\n", what,
            std::chrono::duration<double, std::micro>(now - last).count());
    last = now;
}

dda_status_t ensure_workspace(dda_matrix* K, size_t bytes, cudaStream_t st) {
    if (K->ws_bytes >= bytes) return DDA_OK;
    if (K->graph_engine) {          // its graph has the old workspace pointers baked in
        pcg_graph_free(K->graph_engine);
        K->graph_engine = nullptr;
    }
    if (K->ws) {
        cudaStreamSynchronize(st);
        dev_free(K->ws);
    }
    K->ws = nullptr;
    K->ws_bytes = 0;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->ws), bytes, st));
    K->ws_bytes = bytes;
    return DDA_OK;
}

}  // namespace dda

extern "C" int64_t dda_launch_count(void) { return dda::g_launches.load(); }

extern "C" const char* dda_last_cuda_error(void) { return dda::g_last_err; }

extern "C" const char* dda_status_string(dda_status_t s) {
    switch (s) {
        case DDA_OK: return "DDA_OK";
        case DDA_ERR_ARG: return "DDA_ERR_ARG";
        case DDA_ERR_CUDA: return "DDA_ERR_CUDA";
        case DDA_ERR_OOM: return "DDA_ERR_OOM";
        case DDA_ERR_NOT_SPD: return "DDA_ERR_NOT_SPD";
        case DDA_ERR_BREAKDOWN: return "DDA_ERR_BREAKDOWN";
        case DDA_ERR_NO_CONVERGENCE: return "DDA_ERR_NO_CONVERGENCE";
        case DDA_ERR_NCCL: return "DDA_ERR_NCCL";
    }
    return "DDA_ERR_UNKNOWN";
}
