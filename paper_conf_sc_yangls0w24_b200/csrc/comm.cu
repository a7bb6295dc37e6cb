// comm.cu — the multi-GPU communicator of libxbfs (include/xbfs_dist.h), one
// process per GPU on one node.  Reading R-10: the
// per-level frontier exchange is peer-memory stores fused into the producing
// kernels (CUDA IPC over NVLink/NVSwitch, dist.cu), so what remains collective
// is host-side and tiny: a barrier, the all-reduce of the per-level counters
// (every rank takes the same direction decision, north_star), and small
// all-gathers (counts, IPC handles) during the build.  They run over one POSIX
// shared-memory segment the ranks attach by name; the 128-byte unique id carries
// that name and is broadcast by the caller (torch.distributed), as an ncclUniqueId
// would be.  No CUDA call is made here: the host collectives work (and are
// tested) without a GPU.
#include <errno.h>
#include <fcntl.h>
#include <sched.h>
#include <stdio.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#include <atomic>
#include <new>

#include "common.cuh"
#include "xbfs_dist.h"

namespace xbfs {
namespace comm {

constexpr uint64_t kMagic = 0x58424653434f4d4dull;   // "XBFSCOMM"
constexpr int kSlotBytes = 4096;                       // per-rank exchange slot
constexpr double kTimeoutS = 600.0;                    // a peer that never arrives -> error, not a hang

struct alignas(128) Shared {
    std::atomic<uint64_t> magic;
    std::atomic<int32_t> attached;
    int32_t nranks;
    alignas(128) std::atomic<uint32_t> arrived;        // barrier: arrivals of the current generation
    alignas(128) std::atomic<uint32_t> generation;     // bumped by the last arrival
    alignas(128) unsigned char slot[kMaxCommRanks][kSlotBytes];
};

double now_s() {
    timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return t.tv_sec + 1e-9 * t.tv_nsec;
}

}  // namespace comm
}  // namespace xbfs

using namespace xbfs;
using namespace xbfs::comm;

struct xbfs_comm {
    int rank = 0, nranks = 1;
    char name[64] = {0};
    Shared* sh = nullptr;
    bool owner_unlinked = false;
};

namespace {

xbfs_status barrier_impl(xbfs_comm* c) {
    Shared* sh = c->sh;
    const uint32_t gen = sh->generation.load(std::memory_order_acquire);
    if (sh->arrived.fetch_add(1, std::memory_order_acq_rel) + 1 == (uint32_t)c->nranks) {
        sh->arrived.store(0, std::memory_order_relaxed);
        sh->generation.fetch_add(1, std::memory_order_acq_rel);
        return XBFS_OK;
    }
    const double t0 = now_s();
    int spins = 0;
    while (sh->generation.load(std::memory_order_acquire) == gen) {
        if (++spins > 1000) {
            sched_yield();
            if ((spins & 1023) == 0 && now_s() - t0 > kTimeoutS)
                return set_error(XBFS_ERR_STATE, "xbfs comm: a peer did not reach the barrier within %.0f s",
                                 kTimeoutS);
        }
    }
    return XBFS_OK;
}

}  // namespace

namespace xbfs {

// Collectives used by dist.cu (host side; `bytes` <= kSlotBytes per call).
xbfs_status comm_barrier(xbfs_comm* c) { return c->nranks == 1 ? XBFS_OK : barrier_impl(c); }

xbfs_status comm_allgather(xbfs_comm* c, const void* mine, size_t bytes, void* all) {
    if (bytes > (size_t)kSlotBytes) return set_error(XBFS_ERR_INVALID_ARG, "xbfs comm: all-gather of %zu bytes", bytes);
    if (c->nranks == 1) {
        memcpy(all, mine, bytes);
        return XBFS_OK;
    }
    memcpy(c->sh->slot[c->rank], mine, bytes);
    xbfs_status s = barrier_impl(c);
    if (s != XBFS_OK) return s;
    for (int r = 0; r < c->nranks; ++r) memcpy((char*)all + (size_t)r * bytes, c->sh->slot[r], bytes);
    return barrier_impl(c);   // slots are reused by the next collective
}

xbfs_status comm_allreduce_sum(xbfs_comm* c, const int64_t* in, int64_t* out, int n) {
    if (n * sizeof(int64_t) > (size_t)kSlotBytes) return set_error(XBFS_ERR_INVALID_ARG, "xbfs comm: all-reduce of %d", n);
    if (c->nranks == 1) {
        if (out != in) memcpy(out, in, n * sizeof(int64_t));
        return XBFS_OK;
    }
    memcpy(c->sh->slot[c->rank], in, n * sizeof(int64_t));
    xbfs_status s = barrier_impl(c);
    if (s != XBFS_OK) return s;
    for (int i = 0; i < n; ++i) {
        int64_t t = 0;
        for (int r = 0; r < c->nranks; ++r) t += reinterpret_cast<const int64_t*>(c->sh->slot[r])[i];
        out[i] = t;
    }
    return barrier_impl(c);
}

int comm_rank(const xbfs_comm* c) { return c->rank; }
int comm_size(const xbfs_comm* c) { return c->nranks; }

}  // namespace xbfs

extern "C" {

xbfs_status xbfs_get_unique_id(uint8_t id[XBFS_UNIQUE_ID_BYTES]) {
    if (!id) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_get_unique_id: NULL id");
    memset(id, 0, XBFS_UNIQUE_ID_BYTES);
    uint64_t r = 0;
    FILE* f = fopen("/dev/urandom", "rb");
    if (!f || fread(&r, sizeof(r), 1, f) != 1) r = (uint64_t)now_s() * 6364136223846793005ull ^ (uint64_t)getpid();
    if (f) fclose(f);
    memcpy(id, &kMagic, 8);
    snprintf((char*)id + 8, 64, "/xbfs.%d.%016llx", (int)getpid(), (unsigned long long)r);
    return XBFS_OK;
}

xbfs_status xbfs_comm_init(const uint8_t id[XBFS_UNIQUE_ID_BYTES], int32_t nranks, int32_t rank, xbfs_comm** out) {
    if (!out) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_init: out is NULL");
    *out = nullptr;
    if (!id) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_init: NULL id");
    if (nranks < 1 || nranks > kMaxCommRanks || rank < 0 || rank >= nranks)
        return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_init: rank %d of %d (at most %d ranks)", rank, nranks,
                         kMaxCommRanks);
    uint64_t magic;
    memcpy(&magic, id, 8);
    if (magic != kMagic || id[8] != '/') return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_init: not an xbfs unique id");
    xbfs_comm* c = new (std::nothrow) xbfs_comm();
    if (!c) return set_error(XBFS_ERR_OUT_OF_MEMORY, "host allocation failed");
    c->rank = rank;
    c->nranks = nranks;
    strncpy(c->name, (const char*)id + 8, sizeof(c->name) - 1);
    if (nranks == 1) {   // no peers: no segment
        *out = c;
        return XBFS_OK;
    }
    int fd = -1;
    if (rank == 0) {
        fd = shm_open(c->name, O_CREAT | O_EXCL | O_RDWR, 0600);
        if (fd < 0 || ftruncate(fd, sizeof(Shared)) != 0) {
            if (fd >= 0) close(fd);
            delete c;
            return set_error(XBFS_ERR_STATE, "xbfs_comm_init: shm_open/ftruncate(%s): %s", (const char*)id + 8,
                             strerror(errno));
        }
    } else {
        const double t0 = now_s();
        for (;;) {
            fd = shm_open(c->name, O_RDWR, 0600);
            if (fd >= 0) {
                struct stat st;
                if (fstat(fd, &st) == 0 && st.st_size >= (off_t)sizeof(Shared)) break;
                close(fd);
                fd = -1;
            }
            if (now_s() - t0 > kTimeoutS) {
                delete c;
                return set_error(XBFS_ERR_STATE, "xbfs_comm_init: rank 0's segment %s never appeared", c->name);
            }
            usleep(200);
        }
    }
    void* p = mmap(nullptr, sizeof(Shared), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) {
        delete c;
        return set_error(XBFS_ERR_STATE, "xbfs_comm_init: mmap: %s", strerror(errno));
    }
    c->sh = reinterpret_cast<Shared*>(p);
    if (rank == 0) {
        c->sh->nranks = nranks;                         // the segment is zero-filled by ftruncate
        c->sh->magic.store(kMagic, std::memory_order_release);
    } else {
        const double t0 = now_s();
        while (c->sh->magic.load(std::memory_order_acquire) != kMagic) {
            if (now_s() - t0 > kTimeoutS) {
                munmap(p, sizeof(Shared));
                delete c;
                return set_error(XBFS_ERR_STATE, "xbfs_comm_init: segment %s not initialised", c->name);
            }
            usleep(50);
        }
        if (c->sh->nranks != nranks) {
            munmap(p, sizeof(Shared));
            delete c;
            return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_init: nranks %d differs from rank 0's", nranks);
        }
    }
    c->sh->attached.fetch_add(1, std::memory_order_acq_rel);
    xbfs_status s = barrier_impl(c);
    if (s != XBFS_OK) {
        munmap(p, sizeof(Shared));
        delete c;
        return s;
    }
    if (rank == 0) {        // every rank has mapped it: the name can go (the mapping stays)
        shm_unlink(c->name);
        c->owner_unlinked = true;
    }
    *out = c;
    return XBFS_OK;
}

xbfs_status xbfs_comm_barrier(xbfs_comm* c) {
    if (!c) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_barrier: NULL comm");
    return comm_barrier(c);
}

xbfs_status xbfs_comm_allreduce_i64(xbfs_comm* c, const int64_t* in, int64_t* out, int32_t count) {
    if (!c || !in || !out || count < 0) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_comm_allreduce_i64: bad args");
    return comm_allreduce_sum(c, in, out, count);
}

void xbfs_comm_destroy(xbfs_comm* c) {
    if (!c) return;
    if (c->sh) {
        if (c->rank == 0 && !c->owner_unlinked) shm_unlink(c->name);
        munmap(c->sh, sizeof(Shared));
    }
    delete c;
}

}  // extern "C"
