// Driver-API virtual memory management for replicas shared between processes without CUDA IPC,
// and NVLS multicast objects (NVSwitch): the pieces of §8 row f3's multicast push.
//
// A replica allocated here is a physical allocation (cuMemCreate, exportable as a POSIX file
// descriptor) mapped into this process; the peers import the descriptor and map the same memory
// (the unicast paths: pulls, halo pushes, chunk merges). When the node supports multicast, every
// process binds its replica to one multicast object and maps the object: a store to the multicast
// address (multimem.st) lands in every process's replica through the switch, so the compaction
// pass stores each dirty element once instead of once per peer (L129-135: dirty data to every
// other copy). Entry points come from the runtime's driver entry-point query (no libcuda link).
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>

namespace accmg {
namespace vmm {

struct Phys {                // a physical allocation of this process and its local mapping
    unsigned long long handle = 0;
    void* ptr = nullptr;
    size_t bytes = 0;
};
struct Map {                 // an imported (peer or multicast) handle mapped into this process
    unsigned long long handle = 0;
    void* ptr = nullptr;
    size_t bytes = 0;
};

// True if the driver entry points are present (else *why says which is missing).
bool available(std::string* why);
// Allocation granularity for `bytes` on `device` that also satisfies multicast binding when
// `multicast` (rounded-up size).
size_t round_up(int device, size_t bytes, bool multicast);

int alloc(int device, size_t bytes, Phys* out, std::string* err);         // + local RW mapping
int export_fd(const Phys& p, int* fd, std::string* err);
int import_map(int device, int fd, size_t bytes, Map* out, std::string* err);  // closes fd
void release(Phys* p);
void release(Map* m);                // unmaps and releases an imported handle
void unmap_only(Map* m);             // unmaps a multicast mapping (the object: mc_release)

// Multicast object for `ndev` devices (created by one process, imported by the others).
int mc_probe(int ndev, size_t bytes, std::string* why);                   // 0 = creatable
int mc_create(int ndev, size_t bytes, unsigned long long* mc, std::string* err);
int mc_export_fd(unsigned long long mc, int* fd, std::string* err);
int mc_import(int fd, unsigned long long* mc, std::string* err);            // closes fd
int mc_add_device(unsigned long long mc, int device, std::string* err);
int mc_bind(unsigned long long mc, const Phys& p, std::string* err);
int mc_map(int device, unsigned long long mc, size_t bytes, Map* out, std::string* err);
void mc_release(unsigned long long mc, int device, size_t bytes, bool bound);

}  // namespace vmm
}  // namespace accmg
