#include "bootstrap.h"

#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <sys/socket.h>
#include <sys/stat.h>
#include <sys/un.h>
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

// abstract-namespace socket address of `rank` in the job `name` (no file system entry)
socklen_t sock_addr(const std::string& name, int rank, sockaddr_un* a) {
    std::memset(a, 0, sizeof(*a));
    a->sun_family = AF_UNIX;
    const int n = std::snprintf(a->sun_path + 1, sizeof(a->sun_path) - 1, "%s_fd%d", name.c_str() + 1, rank);
    return (socklen_t)(offsetof(sockaddr_un, sun_path) + 1 + n);
}

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
    // this rank's descriptor-passing socket (listening before the first barrier)
    listen_fd_ = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
    sockaddr_un sa;
    const socklen_t sl = sock_addr(name_, rank, &sa);
    if (listen_fd_ < 0 || bind(listen_fd_, reinterpret_cast<sockaddr*>(&sa), sl) != 0 || listen(listen_fd_, kMaxRanks) != 0) {
        *err = "bootstrap: cannot listen on the descriptor socket";
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

bool Bootstrap::allgather_fds(const int* mine, int n, int* out, std::string* err) {
    if (n < 1 || n > 64) {
        *err = "bootstrap: 1..64 descriptors per rank";
        return false;
    }
    for (int i = 0; i < world_ * n; ++i) out[i] = -1;
    // send to every other rank (its listener queues the connection until it accepts)
    for (int q = 0; q < world_; ++q) {
        if (q == rank_) continue;
        sockaddr_un sa;
        const socklen_t sl = sock_addr(name_, q, &sa);
        int c = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
        const auto t0 = std::chrono::steady_clock::now();
        while (c >= 0 && connect(c, reinterpret_cast<sockaddr*>(&sa), sl) != 0) {
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(60)) {
                ::close(c);
                c = -1;
                break;
            }
            usleep(1000);
        }
        if (c < 0) {
            *err = "bootstrap: cannot connect to a peer's descriptor socket";
            return false;
        }
        int hdr2[2] = {rank_, n};
        iovec iov{hdr2, sizeof(hdr2)};
        char ctl[CMSG_SPACE(sizeof(int) * 64)];
        std::memset(ctl, 0, sizeof(ctl));
        msghdr m{};
        m.msg_iov = &iov;
        m.msg_iovlen = 1;
        m.msg_control = ctl;
        m.msg_controllen = CMSG_SPACE(sizeof(int) * n);
        cmsghdr* cm = CMSG_FIRSTHDR(&m);
        cm->cmsg_level = SOL_SOCKET;
        cm->cmsg_type = SCM_RIGHTS;
        cm->cmsg_len = CMSG_LEN(sizeof(int) * n);
        std::memcpy(CMSG_DATA(cm), mine, sizeof(int) * n);
        const bool sent = sendmsg(c, &m, 0) == (ssize_t)sizeof(hdr2);
        ::close(c);
        if (!sent) {
            *err = "bootstrap: sendmsg of descriptors failed";
            return false;
        }
    }
    // receive one message from every other rank
    for (int k = 0; k < world_ - 1; ++k) {
        const int c = accept(listen_fd_, nullptr, nullptr);
        if (c < 0) {
            *err = "bootstrap: accept on the descriptor socket failed";
            return false;
        }
        int hdr2[2] = {-1, 0};
        iovec iov{hdr2, sizeof(hdr2)};
        char ctl[CMSG_SPACE(sizeof(int) * 64)];
        msghdr m{};
        m.msg_iov = &iov;
        m.msg_iovlen = 1;
        m.msg_control = ctl;
        m.msg_controllen = sizeof(ctl);
        const ssize_t got = recvmsg(c, &m, MSG_CMSG_CLOEXEC);
        ::close(c);
        cmsghdr* cm = CMSG_FIRSTHDR(&m);
        if (got != (ssize_t)sizeof(hdr2) || hdr2[0] < 0 || hdr2[0] >= world_ || hdr2[1] != n || !cm ||
            cm->cmsg_type != SCM_RIGHTS || cm->cmsg_len != CMSG_LEN(sizeof(int) * n)) {
            *err = "bootstrap: malformed descriptor message";
            return false;
        }
        std::memcpy(out + hdr2[0] * n, CMSG_DATA(cm), sizeof(int) * n);
    }
    return barrier(err);
}

void Bootstrap::close() {
    if (listen_fd_ >= 0) {
        ::close(listen_fd_);
        listen_fd_ = -1;
    }
    if (!base_) return;
    Header* H = hdr(base_);
    const bool last = H->closed.fetch_add(1) + 1 == (uint32_t)world_;
    munmap(base_, bytes_);
    base_ = nullptr;
    if (last || rank_ == 0) shm_unlink(name_.c_str());
}

}  // namespace accmg
