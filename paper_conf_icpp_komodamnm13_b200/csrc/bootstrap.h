// Single-node bootstrap for the one-process-per-GPU mode: a POSIX shared-memory segment named
// after the job's unique id gives every rank a host barrier and a small mailbox for exchanging
// CUDA IPC handles (device buffers of peers are then mapped and reached over NVLink / NVSwitch).
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>

namespace accmg {

class Bootstrap {
public:
    static constexpr int kMaxRanks = 64;
    static constexpr size_t kSlotBytes = 16384;

    // Opens (rank 0 creates) the segment for `world` ranks. Returns false (and sets *err) on failure.
    bool open(const uint8_t id[128], int rank, int world, std::string* err);
    void close();
    bool barrier(std::string* err);          // all ranks; times out after 300 s
    void* slot(int rank);                    // mailbox of `rank` (kSlotBytes)
    bool is_open() const { return base_ != nullptr; }
    // All-gather of file descriptors (n per rank, the same n everywhere) over Unix-domain sockets
    // (SCM_RIGHTS): out[q * n + i] = rank q's i-th descriptor, received as a new descriptor here
    // (out[rank * n + i] = -1). Collective; ends with a barrier.
    bool allgather_fds(const int* mine, int n, int* out, std::string* err);

private:
    int listen_fd_ = -1;
    void* base_ = nullptr;
    size_t bytes_ = 0;
    int rank_ = 0, world_ = 1;
    std::string name_;
};

}  // namespace accmg
