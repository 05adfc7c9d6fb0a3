/*
 * fake_nccl.c — TEST SUPPORT ONLY. A stand-in for libnccl exporting the entry
 * points libpepp_spmv.so loads with dlopen (nccl_dl.cpp), so that several
 * processes sharing ONE GPU can run the library's partitioned path (real
 * NCCL refuses two ranks on one device). Semantics follow NCCL's: calls
 * between ncclGroupStart/End are matched in order per peer; a call outside a
 * group is a group of one; point-to-point groups involve only the peers they
 * name (per-pair mailboxes with published / consumed message counters, no
 * barrier), collectives (broadcast, all-reduce) every rank. Data moves
 * through a shared, file-backed mapping with a process-shared barrier for
 * the collectives; the device <-> host copies are synchronous (the stream is
 * synchronised first). MAXR ranks, PEPP_FAKE_NCCL_BOX_MB per pair message. Selected by the
 * library when PEPP_NCCL_LIB points at this .so.
 *
 * Build: gcc -O2 -shared -fPIC fake_nccl.c -I$CUDA/include -L$CUDA/lib64 -lcudart
 */
#include <cuda_runtime.h>
#include <fcntl.h>
#include <sched.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#define EXPORT __attribute__((visibility("default")))
#define MAXR 8
#define MAXOPS 4096

typedef struct { char internal[128]; } ncclUniqueId;

enum { OP_SEND, OP_RECV, OP_BCAST, OP_AR };
typedef struct {
    int kind;
    const void* sbuf;
    void* rbuf;
    size_t bytes;
    int peer;   /* peer or root */
    int dtype, redop;
    size_t count;
    cudaStream_t stream;
} Op;

typedef struct {
    volatile int count;
    volatile int gen;
} Barrier;

typedef struct {
    int rank, nranks;
    char path[160];
    unsigned char* base;
    size_t box;          /* bytes per (src, dst) box and per broadcast root */
    size_t size;
    Op ops[MAXOPS];
    int nops;
} Comm;

typedef Comm* ncclComm_t;
static __thread int g_depth = 0;
static __thread Comm* g_pending = NULL;   /* the communicator with queued ops (one at a time) */

static Barrier* bar(Comm* c) { return (Barrier*)c->base; }
static unsigned char* box(Comm* c, int src, int dst) { return c->base + 4096 + ((size_t)src * MAXR + dst) * c->box; }
static unsigned char* bcast(Comm* c, int root) { return c->base + 4096 + (size_t)MAXR * MAXR * c->box + (size_t)root * c->box; }
#define ARMAX 65536   /* all-reduce payload per rank and group */
static unsigned char* arslot(Comm* c, int r) { return c->base + 4096 + (size_t)MAXR * MAXR * c->box + (size_t)MAXR * c->box + (size_t)r * ARMAX; }

static void barrier(Comm* c) {
    Barrier* b = bar(c);
    int g = __atomic_load_n(&b->gen, __ATOMIC_SEQ_CST);
    if (__atomic_add_fetch(&b->count, 1, __ATOMIC_SEQ_CST) == c->nranks) {
        __atomic_store_n(&b->count, 0, __ATOMIC_SEQ_CST);
        __atomic_store_n(&b->gen, g + 1, __ATOMIC_SEQ_CST);
    } else {
        while (__atomic_load_n(&b->gen, __ATOMIC_SEQ_CST) == g) sched_yield();
    }
}

/* ncclDataType_t: 0/1 int8/uint8, 2/3 int32/uint32, 4/5 int64/uint64, 6 half, 7 float, 8 double, 9 bf16 */
static size_t dsize(int dtype) {
    switch (dtype) {
    case 2: case 3: case 7: return 4;
    case 4: case 5: case 8: return 8;
    case 6: case 9: return 2;
    default: return 1;
    }
}

EXPORT const char* ncclGetErrorString(int r) { return r ? "fake nccl error" : "no error"; }

EXPORT int ncclGetUniqueId(ncclUniqueId* id) {
    memset(id, 0, sizeof(*id));
    struct timespec ts;
    clock_gettime(CLOCK_REALTIME, &ts);
    snprintf(id->internal, sizeof(id->internal), "/tmp/pepp_fake_nccl_%d_%ld", (int)getpid(), (long)ts.tv_nsec);
    return 0;
}

EXPORT int ncclCommInitRank(ncclComm_t* out, int nranks, ncclUniqueId id, int rank) {
    if (nranks < 1 || nranks > MAXR || rank < 0 || rank >= nranks) return 4;
    Comm* c = (Comm*)calloc(1, sizeof(Comm));
    c->rank = rank;
    c->nranks = nranks;
    snprintf(c->path, sizeof(c->path), "%s", id.internal);
    const char* e = getenv("PEPP_FAKE_NCCL_BOX_MB");
    c->box = (size_t)(e ? atoi(e) : 16) << 20;
    c->size = 4096 + (size_t)MAXR * MAXR * c->box + (size_t)MAXR * c->box + (size_t)MAXR * ARMAX;
    int fd = open(c->path, O_RDWR | O_CREAT, 0600);
    if (fd < 0) { free(c); return 2; }
    if (ftruncate(fd, (off_t)c->size) != 0) { close(fd); free(c); return 2; }
    c->base = (unsigned char*)mmap(NULL, c->size, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (c->base == MAP_FAILED) { free(c); return 2; }
    /* rendezvous: a counter of arrivals, then the barrier is usable */
    volatile int* arrived = (volatile int*)(c->base + 1024);
    __atomic_add_fetch(arrived, 1, __ATOMIC_SEQ_CST);
    while (__atomic_load_n(arrived, __ATOMIC_SEQ_CST) < nranks) sched_yield();
    *out = c;
    return 0;
}

EXPORT int ncclCommDestroy(ncclComm_t c) {
    if (!c) return 0;
    barrier(c);
    munmap(c->base, c->size);
    if (c->rank == 0) unlink(c->path);
    free(c);
    return 0;
}

EXPORT int ncclCommGetAsyncError(ncclComm_t c, int* err) { (void)c; *err = 0; return 0; }

/* per (src, dst) mailbox state: messages published / consumed (one message =
   all sends src -> dst of one group, concatenated in call order) */
static volatile int* pub(Comm* c, int src, int dst) { return (volatile int*)(c->base + 3072) + src * MAXR + dst; }
static volatile int* con(Comm* c, int src, int dst) { return (volatile int*)(c->base + 3072 + 256) + src * MAXR + dst; }

static int flush(Comm* c) {
    size_t out[MAXR] = {0}, in[MAXR] = {0}, bc[MAXR] = {0};
    int has_coll = 0, sends_to[MAXR] = {0}, recvs_from[MAXR] = {0};
    for (int i = 0; i < c->nops; ++i) {
        if (cudaStreamSynchronize(c->ops[i].stream) != cudaSuccess) return 1;
        Op* o = &c->ops[i];
        if (o->kind == OP_BCAST || o->kind == OP_AR) has_coll = 1;
        else if (o->kind == OP_SEND) sends_to[o->peer] = 1;
        else recvs_from[o->peer] = 1;
    }
    /* point-to-point: like NCCL, only the two peers take part (no barrier):
       wait until the previous message to that peer was consumed, write, publish */
    for (int q = 0; q < c->nranks; ++q) {
        if (!sends_to[q]) continue;
        while (__atomic_load_n(pub(c, c->rank, q), __ATOMIC_ACQUIRE) != __atomic_load_n(con(c, c->rank, q), __ATOMIC_ACQUIRE))
            sched_yield();
        for (int i = 0; i < c->nops; ++i) {
            Op* o = &c->ops[i];
            if (o->kind != OP_SEND || o->peer != q) continue;
            if (out[q] + o->bytes > c->box) return 3;
            cudaMemcpy(box(c, c->rank, q) + out[q], o->sbuf, o->bytes, cudaMemcpyDeviceToHost);
            out[q] += o->bytes;
        }
        __atomic_add_fetch(pub(c, c->rank, q), 1, __ATOMIC_RELEASE);
    }
    size_t arc = 0;
    if (has_coll) {
        for (int i = 0; i < c->nops; ++i) {            /* collectives, phase 1: publish */
            Op* o = &c->ops[i];
            if (o->kind == OP_BCAST) {
                if (bc[o->peer] + o->bytes > c->box) return 3;
                if (c->rank == o->peer)
                    cudaMemcpy(bcast(c, o->peer) + bc[o->peer], o->sbuf, o->bytes, cudaMemcpyDeviceToHost);
                bc[o->peer] += o->bytes;
            } else if (o->kind == OP_AR) {
                if (arc + o->bytes > ARMAX) return 3;
                cudaMemcpy(arslot(c, c->rank) + arc, o->sbuf, o->bytes, cudaMemcpyDeviceToHost);
                arc += o->bytes;
            }
        }
        barrier(c);
    }
    memset(bc, 0, sizeof(bc));
    arc = 0;
    for (int q = 0; q < c->nranks; ++q) {            /* point-to-point receives, in call order per peer */
        if (!recvs_from[q]) continue;
        while (__atomic_load_n(pub(c, q, c->rank), __ATOMIC_ACQUIRE) == __atomic_load_n(con(c, q, c->rank), __ATOMIC_ACQUIRE))
            sched_yield();
        for (int i = 0; i < c->nops; ++i) {
            Op* o = &c->ops[i];
            if (o->kind != OP_RECV || o->peer != q) continue;
            cudaMemcpy(o->rbuf, box(c, q, c->rank) + in[q], o->bytes, cudaMemcpyHostToDevice);
            in[q] += o->bytes;
        }
        __atomic_add_fetch(con(c, q, c->rank), 1, __ATOMIC_RELEASE);
    }
    for (int i = 0; i < c->nops && has_coll; ++i) {            /* collectives, phase 2: consume */
        Op* o = &c->ops[i];
        if (o->kind == OP_BCAST) {
            if (c->rank != o->peer)
                cudaMemcpy(o->rbuf, bcast(c, o->peer) + bc[o->peer], o->bytes, cudaMemcpyHostToDevice);
            else if (o->rbuf != o->sbuf)
                cudaMemcpy(o->rbuf, o->sbuf, o->bytes, cudaMemcpyDeviceToDevice);
            bc[o->peer] += o->bytes;
        } else if (o->kind == OP_AR) {
            static __thread unsigned char tmp[ARMAX];
            for (size_t k = 0; k < o->count; ++k) {
                double dv = 0; int64_t iv = 0;
                for (int r = 0; r < c->nranks; ++r) {
                    const unsigned char* src = arslot(c, r) + arc + k * dsize(o->dtype);
                    if (o->dtype == 8 || o->dtype == 7) {
                        double v;
                        if (o->dtype == 8) memcpy(&v, src, 8); else { float f; memcpy(&f, src, 4); v = f; }
                        dv = r == 0 ? v : (o->redop == 2 ? (v > dv ? v : dv) : dv + v);
                    }
                    else { int64_t v = 0; memcpy(&v, src, dsize(o->dtype)); iv = r == 0 ? v : (o->redop == 2 ? (v > iv ? v : iv) : iv + v); }
                }
                if (o->dtype == 8) memcpy(tmp + k * 8, &dv, 8);
                else if (o->dtype == 7) { float f = (float)dv; memcpy(tmp + k * 4, &f, 4); }
                else memcpy(tmp + k * dsize(o->dtype), &iv, dsize(o->dtype));
            }
            cudaMemcpy(o->rbuf, tmp, o->bytes, cudaMemcpyHostToDevice);
            arc += o->bytes;
        }
    }
    /* pageable H2D cudaMemcpy may return before its DMA lands: make the data
       visible to work the caller enqueues next on any stream (real NCCL
       orders it on the op's stream) */
    if (cudaDeviceSynchronize() != cudaSuccess) return 1;
    if (has_coll) barrier(c);   /* the collective slots may be reused by the next group */
    c->nops = 0;
    return cudaGetLastError() == cudaSuccess ? 0 : 1;
}

static int flush_checked(Comm* c) {
    int r = flush(c);
    if (r) {
        cudaError_t e = cudaGetLastError();
        fprintf(stderr, "[fake nccl] rank %d/%d: group of %d ops failed (%d; cuda: %s)\n", c->rank, c->nranks, c->nops, r,
                cudaGetErrorString(e));
        c->nops = 0;
    }
    return r;
}

static int enqueue(Comm* c, Op o) {
    if (c->nops >= MAXOPS) return 3;
    c->ops[c->nops++] = o;
    if (g_depth == 0) return flush_checked(c);
    g_pending = c;
    return 0;
}

EXPORT int ncclGroupStart(void) { ++g_depth; return 0; }
EXPORT int ncclGroupEnd(void) {
    if (g_depth <= 0) return 4;
    if (--g_depth == 0 && g_pending) { Comm* c = g_pending; g_pending = NULL; return flush_checked(c); }
    return 0;
}

EXPORT int ncclSend(const void* buf, size_t count, int dtype, int peer, ncclComm_t c, cudaStream_t s) {
    Op o = {OP_SEND, buf, NULL, count * dsize(dtype), peer, dtype, 0, count, s};
    return enqueue(c, o);
}
EXPORT int ncclRecv(void* buf, size_t count, int dtype, int peer, ncclComm_t c, cudaStream_t s) {
    Op o = {OP_RECV, NULL, buf, count * dsize(dtype), peer, dtype, 0, count, s};
    return enqueue(c, o);
}
EXPORT int ncclBroadcast(const void* sbuf, void* rbuf, size_t count, int dtype, int root, ncclComm_t c, cudaStream_t s) {
    Op o = {OP_BCAST, sbuf, rbuf, count * dsize(dtype), root, dtype, 0, count, s};
    return enqueue(c, o);
}
EXPORT int ncclAllReduce(const void* sbuf, void* rbuf, size_t count, int dtype, int op, ncclComm_t c, cudaStream_t s) {
    Op o = {OP_AR, sbuf, rbuf, count * dsize(dtype), 0, dtype, op, count, s};
    return enqueue(c, o);
}
