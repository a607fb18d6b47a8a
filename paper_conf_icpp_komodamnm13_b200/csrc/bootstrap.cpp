#include "bootstrap.h"

#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>

namespace accmg {

namespace {

constexpr uint32_t kMagic = 0xACC0B007u;

struct Header {
    std::atomic<uint32_t> magic;
    std::atomic<uint32_t> count;
    std::atomic<uint32_t> generation;
    std::atomic<uint32_t> closed;
    uint32_t world;
    uint32_t pad[11];
};

Header* hdr(void* base) { return static_cast<Header*>(base); }

}  // namespace

bool Bootstrap::open(const uint8_t id[128], int rank, int world, std::string* err) {
    if (world > kMaxRanks) {
        *err = "bootstrap: too many ranks";
        return false;
    }
    char nm[64];
    uint64_t h = 1469598103934665603ull;  // FNV-1a of the id
    for (int i = 0; i < 128; ++i) h = (h ^ id[i]) * 1099511628211ull;
    std::snprintf(nm, sizeof(nm), "/accmg_%016llx", (unsigned long long)h);
    name_ = nm;
    rank_ = rank;
    world_ = world;
    bytes_ = 4096 + (size_t)kMaxRanks * kSlotBytes;
    int fd = -1;
    const auto t0 = std::chrono::steady_clock::now();
    if (rank == 0) {
        shm_unlink(nm);
        fd = shm_open(nm, O_CREAT | O_EXCL | O_RDWR, 0600);
        if (fd < 0 || ftruncate(fd, (off_t)bytes_) != 0) {
            *err = std::string("bootstrap: cannot create shared memory ") + nm;
            if (fd >= 0) ::close(fd);
            return false;
        }
    } else {
        while ((fd = shm_open(nm, O_RDWR, 0600)) < 0) {
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(300)) {
                *err = std::string("bootstrap: timed out waiting for rank 0 to create ") + nm;
                return false;
            }
            usleep(1000);
        }
        struct stat st;
        while (fstat(fd, &st) == 0 && (size_t)st.st_size < bytes_) usleep(1000);
    }
    base_ = mmap(nullptr, bytes_, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    ::close(fd);
    if (base_ == MAP_FAILED) {
        base_ = nullptr;
        *err = "bootstrap: mmap failed";
        return false;
    }
    Header* H = hdr(base_);
    if (rank == 0) {
        H->count.store(0);
        H->generation.store(0);
        H->closed.store(0);
        H->world = (uint32_t)world;
        H->magic.store(kMagic, std::memory_order_release);
    } else {
        while (H->magic.load(std::memory_order_acquire) != kMagic) {
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(300)) {
                *err = "bootstrap: timed out waiting for the segment header";
                return false;
            }
            usleep(1000);
        }
        if ((int)H->world != world) {
            *err = "bootstrap: world size mismatch between ranks";
            return false;
        }
    }
    return barrier(err);
}

bool Bootstrap::barrier(std::string* err) {
    Header* H = hdr(base_);
    const uint32_t gen = H->generation.load(std::memory_order_acquire);
    if (H->count.fetch_add(1, std::memory_order_acq_rel) + 1 == (uint32_t)world_) {
        H->count.store(0, std::memory_order_relaxed);
        H->generation.store(gen + 1, std::memory_order_release);
        return true;
    }
    const auto t0 = std::chrono::steady_clock::now();
    int spins = 0;
    while (H->generation.load(std::memory_order_acquire) == gen) {
        if (++spins > 1000) {
            sched_yield();
            if ((spins & 1023) == 0 && std::chrono::steady_clock::now() - t0 > std::chrono::seconds(300)) {
                *err = "bootstrap: host barrier timed out (a rank did not make the same collective call)";
                return false;
            }
        }
    }
    return true;
}

void* Bootstrap::slot(int r) { return static_cast<char*>(base_) + 4096 + (size_t)r * kSlotBytes; }

void Bootstrap::close() {
    if (!base_) return;
    Header* H = hdr(base_);
    const bool last = H->closed.fetch_add(1) + 1 == (uint32_t)world_;
    munmap(base_, bytes_);
    base_ = nullptr;
    if (last || rank_ == 0) shm_unlink(name_.c_str());
}

}  // namespace accmg
