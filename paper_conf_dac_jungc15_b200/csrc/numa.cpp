// NUMA placement for multi-GPU host-resident runs.
//
// A B200 node hangs its GPUs off two (or more) CPU sockets.  Host-resident VP buffers are
// read by the GPU's copy engine over PCIe; pages on the far socket cross the inter-socket
// link first, and the worker thread that drives a GPU (executor.cpp, Workers) issues its
// launches and copies fastest from a core near that GPU.  This file finds the GPU's NUMA
// node and local CPUs from sysfs (the PCI device of the GPU's bus id), pins the per-GPU
// worker threads there, and allocates page-locked host memory bound to that node
// (svp_host_alloc): anonymous mmap + mbind(MPOL_PREFERRED) + cudaHostRegister, so the pages
// are faulted in on the GPU's node when CUDA pins them.
//
// Everything degrades to "no placement" (node -1) when sysfs says nothing (single-socket
// hosts report -1, containers may hide /sys/bus/pci): the allocation is still page-locked
// and usable, just not placed.
#include <errno.h>
#include <pthread.h>
#include <sched.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <cuda_runtime.h>

#include <string>

#include "internal.h"

namespace svp {

// sysfs directory of the GPU's PCI function, e.g. /sys/bus/pci/devices/0000:1b:00.0
static std::string pci_dir(int ordinal) {
    char bus[64] = {0};
    if (cudaDeviceGetPCIBusId(bus, sizeof bus, ordinal) != cudaSuccess) {
        cudaGetLastError();
        return "";
    }
    unsigned dom = 0, b = 0, dev = 0, fn = 0;
    if (sscanf(bus, "%x:%x:%x.%x", &dom, &b, &dev, &fn) != 4) return "";
    char path[128];
    snprintf(path, sizeof path, "/sys/bus/pci/devices/%04x:%02x:%02x.%x", dom, b, dev, fn);
    return path;
}

int gpu_numa_node(int ordinal) {
    const std::string dir = pci_dir(ordinal);
    if (dir.empty()) return -1;
    FILE* f = fopen((dir + "/numa_node").c_str(), "r");
    if (!f) return -1;
    int node = -1;
    if (fscanf(f, "%d", &node) != 1) node = -1;
    fclose(f);
    return node;
}

// Parse a cpulist ("0-55,112-167") into a cpu_set_t; false if empty or unreadable.
bool parse_cpulist(const char* s, cpu_set_t* set) {
    CPU_ZERO(set);
    int n = 0;
    while (*s) {
        char* end = nullptr;
        long a = strtol(s, &end, 10);
        if (end == s) break;
        long b = a;
        s = end;
        if (*s == '-') {
            b = strtol(s + 1, &end, 10);
            if (end == s + 1) return false;
            s = end;
        }
        if (a < 0 || b < a) return false;
        for (long c = a; c <= b && c < CPU_SETSIZE; ++c) {
            CPU_SET((int)c, set);
            ++n;
        }
        while (*s == ',' || *s == '\n' || *s == ' ') ++s;
    }
    return n > 0;
}

bool gpu_local_cpus(int ordinal, cpu_set_t* set) {
    const std::string dir = pci_dir(ordinal);
    if (dir.empty()) return false;
    FILE* f = fopen((dir + "/local_cpulist").c_str(), "r");
    if (!f) return false;
    char buf[4096] = {0};
    const size_t got = fread(buf, 1, sizeof buf - 1, f);
    fclose(f);
    buf[got] = 0;
    return parse_cpulist(buf, set);
}

// Pin thread th (a per-GPU worker) to the GPU's local CPUs, intersected with the CPUs this
// process may run on.  SVP_NUMA_AFFINITY=0 disables it.  Returns true if pinned.
bool pin_thread_near_gpu(int ordinal, pthread_t th) {
    const char* env = getenv("SVP_NUMA_AFFINITY");
    if (env && env[0] == '0') return false;
    cpu_set_t local, allowed;
    if (!gpu_local_cpus(ordinal, &local)) return false;
    if (sched_getaffinity(0, sizeof allowed, &allowed) != 0) return false;
    cpu_set_t both;
    CPU_AND(&both, &local, &allowed);
    if (CPU_COUNT(&both) == 0) return false;
    return pthread_setaffinity_np(th, sizeof both, &both) == 0;
}

// mmap + mbind(MPOL_PREFERRED, node) + cudaHostRegister.  *node_out = the node the pages were
// bound to, or -1 (no placement).  len is rounded up to whole pages by the caller.
svp_status host_alloc_near(int ordinal, size_t len, void** out, int* node_out, std::string* err) {
    *out = nullptr;
    *node_out = -1;
    void* p = mmap(nullptr, len, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (p == MAP_FAILED) {
        *err = std::string("svp_host_alloc: mmap failed: ") + strerror(errno);
        return SVP_E_NOMEM;
    }
    const int node = gpu_numa_node(ordinal);
    if (node >= 0 && node < 1024) {
        unsigned long mask[1024 / (8 * sizeof(unsigned long))] = {0};
        mask[node / (8 * sizeof(unsigned long))] |= 1UL << (node % (8 * sizeof(unsigned long)));
        const long MPOL_PREFERRED_ = 1;  // <numaif.h> is not in the image
        if (syscall(SYS_mbind, p, len, MPOL_PREFERRED_, mask, 1024UL, 0UL) == 0) *node_out = node;
    }
    // pinning faults every page in (now, under the policy above)
    cudaError_t ce = cudaHostRegister(p, len, cudaHostRegisterPortable);
    if (ce != cudaSuccess) {
        cudaGetLastError();
        munmap(p, len);
        *node_out = -1;
        *err = std::string("svp_host_alloc: cudaHostRegister: ") + cudaGetErrorString(ce);
        return ce == cudaErrorMemoryAllocation ? SVP_E_NOMEM : SVP_E_CUDA;
    }
    *out = p;
    return SVP_OK;
}

void host_free_near(void* p, size_t len) {
    cudaHostUnregister(p);
    cudaGetLastError();
    munmap(p, len);
}

}  // namespace svp
