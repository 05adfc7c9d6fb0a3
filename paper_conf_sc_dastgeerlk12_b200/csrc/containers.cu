// containers.cu — smart containers (include/pepp_spmv.h "smart containers").
//
// Paper §IV-D (P@20045–21195): a container keeps copies of its payload on
// several memory units with a valid / outdated state each, and copies data
// only when an access needs it; Fig. 3 (P@22400–26903) walks one vector
// through write / host read / readwrite / read / read / host write and counts
// 2 copies instead of 7. The state machine below is that protocol for one
// host master copy and one device copy; PEPP_DEVICE_SIMULATED runs the same
// state machine without CUDA (counters only) so the protocol is testable on a
// machine without a GPU.
//
// Inter-call parallelism (paper §IV-E P@21908–27091): the
// container also records, per device access, an event on the caller's stream
// — the latest writer, and the readers since that write. A device access on
// any stream first waits (cudaStreamWaitEvent) for what its mode conflicts
// with: READ after the last write (RAW), WRITE after the last write and after
// every reader since (WAW, WAR). Calls on different streams are thus ordered
// by their data dependencies alone, and read-only calls on one vector run
// concurrently (Fig. 3, lines 10 and 12).
#include "pepp_internal.h"

#include <cuda_runtime.h>

#include <cstdlib>
#include <new>

struct pepp_vector_s {
    int64_t n = 0;
    double* host = nullptr;
    bool own_host = false;
    bool pinned = false;
    double* dev = nullptr;
    int device = 0;
    bool simulated = false;
    bool host_valid = true;    // the master copy starts valid
    bool dev_valid = false;
    cudaEvent_t last_use = nullptr;   // end of the latest device work on the vector
    bool has_use = false;
    int64_t h2d = 0, d2h = 0, bytes = 0;
    // dependency tracking (inter-call parallelism)
    static constexpr int kMaxReaders = 16;
    cudaEvent_t writer = nullptr;         // end of the latest writing access
    bool has_writer = false;
    cudaEvent_t readers[kMaxReaders] = {};
    int nreaders = 0;                     // readers since the latest write
    int32_t pending_mode = 0;             // mode of the access being released
    int64_t waits = 0;                    // cross-stream dependency waits inserted
};

namespace {

// works on the vector's device, restores the caller's current device
struct DevScope {
    int prev = -1;
    explicit DevScope(const pepp_vector_t* v);
    ~DevScope() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
        (void)cudaGetLastError();
    }
};

inline bool reads(int32_t m) { return (m & PEPP_ACCESS_READ) != 0; }
inline bool writes(int32_t m) { return (m & PEPP_ACCESS_WRITE) != 0; }
inline bool valid_mode(int32_t m) { return m == PEPP_ACCESS_READ || m == PEPP_ACCESS_WRITE || m == PEPP_ACCESS_READWRITE; }

pepp_status_t wait_device(pepp_vector_t* v) {
    if (v->simulated) return PEPP_OK;
    bool ok = true;
    if (v->has_writer) ok &= cudaEventSynchronize(v->writer) == cudaSuccess;
    for (int i = 0; i < v->nreaders; ++i) ok &= cudaEventSynchronize(v->readers[i]) == cudaSuccess;
    if (v->has_use) ok &= cudaEventSynchronize(v->last_use) == cudaSuccess;
    if (!ok) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    return PEPP_OK;
}

// make `stream` wait for the accesses `mode` conflicts with
pepp_status_t order_after(pepp_vector_t* v, int32_t mode, cudaStream_t stream) {
    if (v->simulated) return PEPP_OK;
    bool ok = true;
    if (v->has_writer) { ok &= cudaStreamWaitEvent(stream, v->writer, 0) == cudaSuccess; ++v->waits; }   // RAW / WAW
    if (writes(mode))
        for (int i = 0; i < v->nreaders; ++i) { ok &= cudaStreamWaitEvent(stream, v->readers[i], 0) == cudaSuccess; ++v->waits; }  // WAR
    if (!ok) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    return PEPP_OK;
}

__global__ void scale_kernel(int64_t n, double alpha, double* __restrict__ v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        v[i] = alpha * v[i];
}

DevScope::DevScope(const pepp_vector_t* v) {
    if (v->simulated) return;
    if (cudaGetDevice(&prev) != cudaSuccess) { (void)cudaGetLastError(); prev = -1; }
    if (prev != v->device) cudaSetDevice(v->device);
}

}  // namespace

extern "C" PEPP_API pepp_status_t pepp_vector_create(int64_t n, double* host, int32_t device, pepp_vector_t** out) {
    if (!out || n < 0) return PEPP_E_INVALID;
    *out = nullptr;
    pepp_vector_t* v = new (std::nothrow) pepp_vector_t();
    if (!v) return PEPP_E_NOMEM;
    v->n = n;
    v->simulated = device == PEPP_DEVICE_SIMULATED;
    if (!v->simulated) {
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) { (void)cudaGetLastError(); delete v; return PEPP_E_CUDA; }
        if (device >= 0) {
            if (device >= ndev) { delete v; return PEPP_E_INVALID; }
            v->device = device;
        } else if (cudaGetDevice(&v->device) != cudaSuccess) {
            (void)cudaGetLastError();
            delete v;
            return PEPP_E_CUDA;
        }
        DevScope scope(v);
        bool ok = cudaEventCreateWithFlags(&v->last_use, cudaEventDisableTiming) == cudaSuccess &&
                  cudaEventCreateWithFlags(&v->writer, cudaEventDisableTiming) == cudaSuccess;
        for (int i = 0; ok && i < pepp_vector_t::kMaxReaders; ++i)
            ok = cudaEventCreateWithFlags(&v->readers[i], cudaEventDisableTiming) == cudaSuccess;
        if (!ok) {
            (void)cudaGetLastError();
            pepp_vector_destroy(v);
            return PEPP_E_CUDA;
        }
    }
    if (host) {
        v->host = host;
    } else {
        v->own_host = true;
        if (!v->simulated && n > 0 && cudaMallocHost((void**)&v->host, sizeof(double) * n) == cudaSuccess) {
            v->pinned = true;
        } else {
            (void)cudaGetLastError();
            v->host = (double*)std::calloc(n > 0 ? n : 1, sizeof(double));
            if (!v->host) { pepp_vector_destroy(v); return PEPP_E_NOMEM; }
        }
    }
    *out = v;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_destroy(pepp_vector_t* v) {
    if (!v) return PEPP_OK;
    DevScope scope(v);
    if (!v->simulated) {
        (void)wait_device(v);
        if (v->dev) cudaFree(v->dev);
        if (v->last_use) cudaEventDestroy(v->last_use);
        if (v->writer) cudaEventDestroy(v->writer);
        for (auto& e : v->readers) if (e) cudaEventDestroy(e);
    }
    if (v->own_host) {
        if (v->pinned) cudaFreeHost(v->host);
        else std::free(v->host);
    }
    delete v;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_acquire_host(pepp_vector_t* v, int32_t mode, double** host) {
    if (!v || !valid_mode(mode)) return PEPP_E_INVALID;
    DevScope scope(v);
    // element-wise access through the [] proxies: any host access needs the
    // latest data, and a host write must not race device work that reads it
    pepp_status_t s = wait_device(v);
    if (s) return s;
    if (!v->host_valid) {
        if (!v->simulated && v->n > 0 &&
            cudaMemcpy(v->host, v->dev, sizeof(double) * v->n, cudaMemcpyDeviceToHost) != cudaSuccess) {
            (void)cudaGetLastError();
            return PEPP_E_CUDA;
        }
        v->d2h += 1;
        v->bytes += (int64_t)sizeof(double) * v->n;
        v->host_valid = true;
    }
    if (writes(mode)) v->dev_valid = false;
    if (host) *host = v->host;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_acquire_device(pepp_vector_t* v, int32_t mode, void* stream, double** dev) {
    if (!v || !valid_mode(mode)) return PEPP_E_INVALID;
    DevScope scope(v);
    if (!v->simulated) {
        if (!v->dev) {
            if (cudaMalloc((void**)&v->dev, sizeof(double) * (v->n > 0 ? v->n : 1)) != cudaSuccess) {
                (void)cudaGetLastError();
                return PEPP_E_NOMEM;
            }
        }
    }
    {
        pepp_status_t so = order_after(v, mode, (cudaStream_t)stream);
        if (so) return so;
    }
    v->pending_mode = mode;
    if (reads(mode) && !v->dev_valid) {
        if (!v->host_valid) return PEPP_E_STATE;   // no valid copy anywhere (cannot happen through this API)
        if (!v->simulated && v->n > 0 &&
            cudaMemcpyAsync(v->dev, v->host, sizeof(double) * v->n, cudaMemcpyHostToDevice, (cudaStream_t)stream) !=
                cudaSuccess) {
            (void)cudaGetLastError();
            return PEPP_E_CUDA;
        }
        v->h2d += 1;
        v->bytes += (int64_t)sizeof(double) * v->n;
        // the copy in writes the device copy: later accesses on other streams
        // must order after it
        if (!v->simulated) {
            if (cudaEventRecord(v->writer, (cudaStream_t)stream) != cudaSuccess) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
            v->has_writer = true;
            v->nreaders = 0;
        }
    }
    // write-only: no copy in, only the allocation ("just a memory allocation
    // is made in the device memory where data is written", P@23793)
    v->dev_valid = true;
    if (writes(mode)) v->host_valid = false;
    if (dev) *dev = v->dev;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_release_device(pepp_vector_t* v, void* stream) {
    if (!v) return PEPP_E_INVALID;
    if (v->simulated) return PEPP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    bool ok = cudaEventRecord(v->last_use, st) == cudaSuccess;
    if (writes(v->pending_mode)) {
        ok &= cudaEventRecord(v->writer, st) == cudaSuccess;
        v->has_writer = true;
        v->nreaders = 0;
    } else if (v->nreaders < pepp_vector_t::kMaxReaders) {
        ok &= cudaEventRecord(v->readers[v->nreaders++], st) == cudaSuccess;
    } else {
        // too many concurrent readers to track: fold them into one by making
        // this stream wait for all of them, then record a single reader
        for (int i = 0; i < v->nreaders; ++i) ok &= cudaStreamWaitEvent(st, v->readers[i], 0) == cudaSuccess;
        ok &= cudaEventRecord(v->readers[0], st) == cudaSuccess;
        v->nreaders = 1;
    }
    v->pending_mode = 0;
    if (!ok) { (void)cudaGetLastError(); return PEPP_E_CUDA; }
    v->has_use = true;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_counters(const pepp_vector_t* v, int64_t* h2d, int64_t* d2h, int64_t* bytes) {
    if (!v) return PEPP_E_INVALID;
    if (h2d) *h2d = v->h2d;
    if (d2h) *d2h = v->d2h;
    if (bytes) *bytes = v->bytes;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_state(const pepp_vector_t* v, int32_t* host_valid, int32_t* device_valid) {
    if (!v) return PEPP_E_INVALID;
    if (host_valid) *host_valid = v->host_valid ? 1 : 0;
    if (device_valid) *device_valid = v->dev_valid ? 1 : 0;
    return PEPP_OK;
}

extern "C" PEPP_API pepp_status_t pepp_vector_scale(pepp_vector_t* v, double alpha, void* stream) {
    if (!v) return PEPP_E_INVALID;
    double* d = nullptr;
    pepp_status_t s = pepp_vector_acquire_device(v, PEPP_ACCESS_READWRITE, stream, &d);
    if (s) return s;
    if (!v->simulated && v->n > 0) {
        const int64_t blocks = (v->n + 255) / 256;
        scale_kernel<<<(int)(blocks < 4096 ? blocks : 4096), 256, 0, (cudaStream_t)stream>>>(v->n, alpha, d);
        if (cudaGetLastError() != cudaSuccess) return PEPP_E_CUDA;
    }
    return pepp_vector_release_device(v, stream);
}

namespace pepp {
int64_t vector_length(const pepp_vector_t* v) { return v ? v->n : -1; }
bool vector_simulated(const pepp_vector_t* v) { return v && v->simulated; }
}  // namespace pepp
