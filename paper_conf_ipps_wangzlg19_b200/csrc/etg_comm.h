// etg_comm.h -- host side of the multi-GPU communicator (etg_comm_* in include/etg.h).
//
// One process (or thread) per GPU partition on ONE node.  The communicator is
// only the control plane: a POSIX shared-memory segment named after the
// 128-byte unique id, holding one slot per rank (pid, device, the CUDA-IPC
// handle of the rank's workspace, its owned range, small all-gather payloads)
// and a sense-reversing host barrier.  The data plane -- the per-iteration
// exchange of SURVEY 8(e) -- is done by the library's own kernels writing into
// the peers' device memory (CUDA-IPC-mapped, over NVLink / NVSwitch between
// GPUs), so no collective library sits on the data path.
//
// The barrier waits with a deadline (ETG_COMM_TIMEOUT_S, default 600 s) and
// checks every second that the peers' processes are still alive, so a dead
// or mismatched rank becomes ETG_ENCCL instead of a hang.
#pragma once
#include <errno.h>
#include <fcntl.h>
#include <sched.h>
#include <signal.h>
#include <stdint.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#include <string>

namespace etg {

constexpr uint32_t kCommMaxRanks = 8;          // = kMaxPeer of the kernels
constexpr uint64_t kCommMagic = 0x45544743'4f4d4d31ull;   // "ETGCOMM1"
constexpr int kCommIdBytes = 128;
constexpr int kCommVals = 16;

struct CommSlot {
    int32_t pid;
    int32_t device;
    uint8_t ipc[64];            // cudaIpcMemHandle_t of the allocation holding the workspace
    uint64_t ipc_off;           // workspace offset inside that allocation
    uint64_t ws_ptr;            // raw workspace pointer (usable by peers in the same process)
    uint64_t val[kCommVals];    // small all-gather payloads
    uint8_t pad[56];
};

struct CommShared {
    uint64_t magic;
    uint32_t world;
    uint32_t joined;            // ranks that opened the segment
    uint32_t bar_count;         // barrier arrivals of the current generation
    uint32_t bar_gen;           // barrier generation
    uint32_t pad[10];
    CommSlot slot[kCommMaxRanks];
};

struct Comm {
    int rank = 0, world = 1, device = -1;
    CommShared *sh = nullptr;
    double timeout_s = 600.0;
    std::string name;
};

inline double comm_now() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}

inline std::string comm_shm_name(const uint8_t *id) {
    static const char *hex = "0123456789abcdef";
    std::string s = "/etg_";
    for (int i = 8; i < 32; ++i) {
        s += hex[id[i] >> 4];
        s += hex[id[i] & 15];
    }
    return s;
}

// 0 = ok; -1 = timeout; -2 = a peer process died
inline int comm_wait_peers_alive(const Comm &c) {
    for (int q = 0; q < c.world; ++q) {
        const int32_t pid = __atomic_load_n(&c.sh->slot[q].pid, __ATOMIC_ACQUIRE);
        if (pid > 0 && pid != getpid() && kill(pid, 0) != 0 && errno == ESRCH) return -2;
    }
    return 0;
}

// Sense-reversing barrier over the shared segment.  Returns 0, -1 (timeout)
// or -2 (peer died).
inline int comm_barrier(const Comm &c) {
    if (c.world <= 1) return 0;
    CommShared *sh = c.sh;
    const uint32_t gen = __atomic_load_n(&sh->bar_gen, __ATOMIC_ACQUIRE);
    if (__atomic_add_fetch(&sh->bar_count, 1u, __ATOMIC_ACQ_REL) == (uint32_t)c.world) {
        __atomic_store_n(&sh->bar_count, 0u, __ATOMIC_RELAXED);
        __atomic_store_n(&sh->bar_gen, gen + 1, __ATOMIC_RELEASE);
        return 0;
    }
    const double t0 = comm_now();
    double next_check = t0 + 1.0;
    for (uint64_t spin = 0;; ++spin) {
        if (__atomic_load_n(&sh->bar_gen, __ATOMIC_ACQUIRE) != gen) return 0;
        if (spin > 4096) sched_yield();
        if ((spin & 1023) == 0) {
            const double t = comm_now();
            if (t - t0 > c.timeout_s) return -1;
            if (t > next_check) {
                next_check = t + 1.0;
                if (comm_wait_peers_alive(c)) return -2;
            }
        }
    }
}

// Open (create on first use) the segment of `id`, take slot `rank`, wait for
// all `world` ranks.  Returns an empty string or an error message; *bad_arg
// tells a caller error (ETG_EINVAL) from a transport one (ETG_ENCCL).
inline std::string comm_open(Comm &c, const uint8_t *id, int rank, int world, int device, bool *bad_arg) {
    uint64_t magic = 0;
    memcpy(&magic, id, 8);
    *bad_arg = true;
    if (magic != kCommMagic) return "not an etg_comm_unique_id";
    if (world < 1 || world > (int)kCommMaxRanks) return "world must be 1..8";
    if (rank < 0 || rank >= world) return "rank must be in [0, world)";
    c.rank = rank;
    c.world = world;
    c.device = device;
    if (const char *t = getenv("ETG_COMM_TIMEOUT_S")) c.timeout_s = atof(t) > 0 ? atof(t) : c.timeout_s;
    c.name = comm_shm_name(id);
    *bad_arg = false;
    const int fd = shm_open(c.name.c_str(), O_CREAT | O_RDWR, 0600);
    if (fd < 0) return std::string("shm_open: ") + strerror(errno);
    if (ftruncate(fd, sizeof(CommShared)) != 0) {
        const int e = errno;
        close(fd);
        return std::string("ftruncate: ") + strerror(e);
    }
    void *p = mmap(nullptr, sizeof(CommShared), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) return std::string("mmap: ") + strerror(errno);
    c.sh = static_cast<CommShared *>(p);
    CommShared *sh = c.sh;
    uint32_t expect = 0;
    if (!__atomic_compare_exchange_n(&sh->world, &expect, (uint32_t)world, false, __ATOMIC_ACQ_REL,
                                     __ATOMIC_ACQUIRE) && expect != (uint32_t)world) {
        *bad_arg = true;
        return "ranks disagree on the world size";
    }
    int32_t none = 0;
    if (!__atomic_compare_exchange_n(&sh->slot[rank].pid, &none, (int32_t)getpid(), false, __ATOMIC_ACQ_REL,
                                     __ATOMIC_ACQUIRE)) {
        *bad_arg = true;
        return "rank slot already taken";
    }
    sh->slot[rank].device = device;
    __atomic_store_n(&sh->magic, kCommMagic, __ATOMIC_RELEASE);
    const uint32_t joined = __atomic_add_fetch(&sh->joined, 1u, __ATOMIC_ACQ_REL);
    if (joined > (uint32_t)world) return "more ranks than world joined this id";
    const double t0 = comm_now();
    double next_check = t0 + 1.0;
    for (uint64_t spin = 0; __atomic_load_n(&sh->joined, __ATOMIC_ACQUIRE) < (uint32_t)world; ++spin) {
        if (spin > 4096) sched_yield();
        if ((spin & 1023) == 0) {
            const double t = comm_now();
            if (t - t0 > c.timeout_s || (t > next_check && comm_wait_peers_alive(c))) {
                shm_unlink(c.name.c_str());          // best effort: no stale segment left behind
                return t - t0 > c.timeout_s ? "timed out waiting for the other ranks to join"
                                            : "a peer process died while joining";
            }
            if (t > next_check) next_check = t + 1.0;
        }
    }
    // everyone has the segment mapped: its name is no longer needed
    if (rank == 0) shm_unlink(c.name.c_str());
    return std::string();
}

inline void comm_close(Comm &c) {
    if (c.sh) munmap(c.sh, sizeof(CommShared));
    c.sh = nullptr;
}

}  // namespace etg
