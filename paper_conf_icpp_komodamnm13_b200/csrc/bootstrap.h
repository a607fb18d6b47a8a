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

private:
    void* base_ = nullptr;
    size_t bytes_ = 0;
    int rank_ = 0, world_ = 1;
    std::string name_;
};

}  // namespace accmg
