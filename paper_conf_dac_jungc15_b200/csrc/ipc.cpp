// ipc.cpp -- cross-process front end: the paper's IPC Manager ("allows
// the virtual embedded GPUs and the host GPU to communicate through an IPC method such
// as socket or shared memory") feeding the Job Queue.
//
// One POSIX shared-memory segment per server:
//   [IpcHeader][IpcSlot x nslots][data arena]
// VP processes (clients, no CUDA needed) bump-allocate their buffers in the arena, write
// inputs there, and submit jobs through a ticketed slot ring; the server thread turns
// every slot into an svp_submit with HOST_PINNED buffers (the arena is cudaHostRegister'ed
// in the server), the context's continuous dispatcher coalesces what many VPs submit,
// and the server marks each slot DONE when svp's completion watermark passes its job --
// the client's svp_ipc_wait then returns and its outputs are in the arena.
//
// Slot protocol (lock-free, wait via polling): slot i starts with ticket i, FREE.  A
// client takes ticket t (fetch_add), waits until slot[t % n] holds ticket t and is FREE,
// writes the job, sets SUBMITTED.  The server consumes tickets in order, submits, later
// sets DONE + status.  The client reads the status, then recycles the slot for ticket
// t + n (ticket += n, FREE).
#include <fcntl.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <deque>
#include <string>
#include <thread>

#include "internal.h"

namespace svp {

static const uint64_t kIpcMagic = 0x5356504950433031ull;  // "SVPIPC01"

enum : uint32_t { SLOT_FREE = 0, SLOT_SUBMITTED = 2, SLOT_DONE = 3 };

struct IpcBuf {
    uint64_t off, bytes;
    int32_t dir, _pad;
};

struct alignas(64) IpcSlot {
    std::atomic<uint64_t> ticket;
    std::atomic<uint32_t> state;
    int32_t status;
    int32_t vp, kernel, nbufs;
    uint32_t args_bytes;
    uint8_t args[SVP_MAX_ARGS];
    IpcBuf bufs[SVP_MAX_BUFS];
};

struct alignas(64) IpcHeader {
    uint64_t magic;
    uint64_t nslots;
    uint64_t slots_off, arena_off, arena_bytes, total_bytes;
    std::atomic<uint64_t> next_ticket;
    std::atomic<uint64_t> arena_head;
    std::atomic<uint32_t> alive;
};
static_assert(std::atomic<uint64_t>::is_always_lock_free, "shared-memory atomics must be lock-free");

static uint64_t align_up64(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

static void pause_briefly(int spins) {
    if (spins < 64) return;
    struct timespec ts{0, spins < 1024 ? 2000 : 20000};
    nanosleep(&ts, nullptr);
}

struct IpcServer {
    Ctx* c = nullptr;
    std::string name;
    int fd = -1;
    uint8_t* base = nullptr;
    uint64_t total = 0;
    IpcHeader* hdr = nullptr;
    IpcSlot* slots = nullptr;
    uint8_t* arena = nullptr;
    bool registered = false;
    std::thread th;
    std::atomic<bool> stop{false};
    std::atomic<uint64_t> served{0};
};

struct IpcClient {
    int fd = -1;
    uint8_t* base = nullptr;
    uint64_t total = 0;
    IpcHeader* hdr = nullptr;
    IpcSlot* slots = nullptr;
    uint8_t* arena = nullptr;
};

// Server-side helpers implemented in executor.cpp
svp_status executor_register_host(Executor* e, void* p, uint64_t bytes, std::string* why);
void executor_unregister_host(Executor* e, void* p);

static void server_loop(IpcServer* s) {
    const uint64_t n = s->hdr->nslots;
    uint64_t next = 0;
    std::deque<std::pair<uint64_t, uint64_t>> pending;  // (ticket, job id), submission order
    int spins = 0;
    while (!s->stop.load(std::memory_order_acquire)) {
        bool progress = false;
        // 1) consume submitted slots in ticket order
        for (int burst = 0; burst < 256; ++burst) {
            IpcSlot& sl = s->slots[next % n];
            if (sl.ticket.load(std::memory_order_acquire) != next ||
                sl.state.load(std::memory_order_acquire) != SLOT_SUBMITTED)
                break;
            svp_job_desc d;
            memset(&d, 0, sizeof(d));
            d.vp = sl.vp;
            d.kernel = sl.kernel;
            d.nbufs = sl.nbufs;
            d.args_bytes = sl.args_bytes;
            svp_status st = SVP_OK;
            if (d.nbufs < 0 || d.nbufs > SVP_MAX_BUFS || d.args_bytes > SVP_MAX_ARGS) st = SVP_E_INVAL;
            if (st == SVP_OK) {
                memcpy(d.args, sl.args, d.args_bytes);
                for (int b = 0; b < d.nbufs; ++b) {
                    const IpcBuf& ib = sl.bufs[b];
                    if (ib.off > s->hdr->arena_bytes || ib.bytes > s->hdr->arena_bytes - ib.off) {
                        st = SVP_E_INVAL;
                        break;
                    }
                    d.bufs[b].ptr = ib.bytes ? (void*)(s->arena + ib.off) : nullptr;
                    d.bufs[b].bytes = ib.bytes;
                    d.bufs[b].dir = ib.dir;
                    d.bufs[b].mem = SVP_MEM_HOST_PINNED;
                }
            }
            uint64_t id = 0;
            if (st == SVP_OK) st = ctx_submit_one(s->c, d, &id);
            if (st != SVP_OK) {
                sl.status = st;
                sl.state.store(SLOT_DONE, std::memory_order_release);
            } else {
                pending.emplace_back(next, id);
            }
            ++next;
            progress = true;
        }
        // 2) complete slots whose jobs the context has finished
        if (!pending.empty()) {
            const uint64_t upto = ctx_completed_upto(s->c);
            while (!pending.empty() && pending.front().second <= upto) {
                IpcSlot& sl = s->slots[pending.front().first % n];
                sl.status = ctx_job_status(s->c, pending.front().second);
                sl.state.store(SLOT_DONE, std::memory_order_release);
                pending.pop_front();
                s->served.fetch_add(1);
                progress = true;
            }
        }
        spins = progress ? 0 : spins + 1;
        pause_briefly(spins);
    }
}

static svp_status map_segment(const char* name, bool create, uint64_t total, int* fd_out, uint8_t** base_out) {
    std::string nm = std::string("/") + name;
    int fd = create ? shm_open(nm.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600) : shm_open(nm.c_str(), O_RDWR, 0600);
    if (fd < 0) {
        set_error(std::string("shm_open(") + nm + ") failed: " + strerror(errno));
        return create ? SVP_E_STATE : SVP_E_INVAL;
    }
    if (create && ftruncate(fd, (off_t)total) != 0) {
        set_error(std::string("ftruncate failed: ") + strerror(errno));
        close(fd);
        shm_unlink(nm.c_str());
        return SVP_E_NOMEM;
    }
    if (!create) {
        struct stat stt;
        if (fstat(fd, &stt) != 0 || (uint64_t)stt.st_size < sizeof(IpcHeader)) {
            set_error("svp_ipc_connect: segment too small");
            close(fd);
            return SVP_E_INVAL;
        }
        total = (uint64_t)stt.st_size;
    }
    void* p = mmap(nullptr, total, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    if (p == MAP_FAILED) {
        set_error(std::string("mmap failed: ") + strerror(errno));
        close(fd);
        if (create) shm_unlink(nm.c_str());
        return SVP_E_NOMEM;
    }
    *fd_out = fd;
    *base_out = (uint8_t*)p;
    return SVP_OK;
}

}  // namespace svp

using namespace svp;

extern "C" {

svp_status svp_ipc_serve(svp_ctx* h, const char* name, uint64_t arena_bytes, int32_t nslots,
                         svp_ipc_server** out) {
    try {
        if (!h || !name || !*name || strchr(name, '/') || !out || nslots < 1 || nslots > (1 << 20) || !arena_bytes) {
            set_error("svp_ipc_serve: bad arguments");
            return SVP_E_INVAL;
        }
        *out = nullptr;
        IpcServer* s = new IpcServer();
        s->c = reinterpret_cast<Ctx*>(h);
        s->name = name;
        const uint64_t slots_off = align_up64(sizeof(IpcHeader), 4096);
        const uint64_t arena_off = align_up64(slots_off + sizeof(IpcSlot) * (uint64_t)nslots, 4096);
        s->total = arena_off + align_up64(arena_bytes, 4096);
        svp_status st = map_segment(name, true, s->total, &s->fd, &s->base);
        if (st) {
            delete s;
            return st;
        }
        s->hdr = new (s->base) IpcHeader();
        s->hdr->nslots = (uint64_t)nslots;
        s->hdr->slots_off = slots_off;
        s->hdr->arena_off = arena_off;
        s->hdr->arena_bytes = arena_bytes;
        s->hdr->total_bytes = s->total;
        s->hdr->next_ticket.store(0);
        s->hdr->arena_head.store(0);
        s->slots = reinterpret_cast<IpcSlot*>(s->base + slots_off);
        for (int32_t i = 0; i < nslots; ++i) {
            IpcSlot* sl = new (&s->slots[i]) IpcSlot();
            sl->ticket.store((uint64_t)i);
            sl->state.store(SLOT_FREE);
        }
        s->arena = s->base + arena_off;
        if (s->c->exec) {
            std::string why;
            if (executor_register_host(s->c->exec, s->arena, arena_bytes, &why) != SVP_OK) {
                set_error("svp_ipc_serve: cudaHostRegister of the arena failed: " + why);
                munmap(s->base, s->total);
                close(s->fd);
                shm_unlink((std::string("/") + name).c_str());
                delete s;
                return SVP_E_CUDA;
            }
            s->registered = true;
        }
        {
            bool running;
            {
                std::lock_guard<std::mutex> lk(s->c->qmu);
                running = s->c->disp_running;
            }
            if (!running) svp_start_dispatcher(h, 50, 0);  // jobs from the ring must get flushed
        }
        s->hdr->magic = kIpcMagic;  // last: clients check it
        s->hdr->alive.store(1, std::memory_order_release);
        s->th = std::thread(server_loop, s);
        *out = reinterpret_cast<svp_ipc_server*>(s);
        return SVP_OK;
    } catch (...) {
        set_error("svp_ipc_serve: internal error");
        return SVP_E_STATE;
    }
}

svp_status svp_ipc_server_stats(svp_ipc_server* hs, uint64_t* served, uint64_t* tickets) {
    if (!hs) {
        set_error("null server");
        return SVP_E_INVAL;
    }
    IpcServer* s = reinterpret_cast<IpcServer*>(hs);
    if (served) *served = s->served.load();
    if (tickets) *tickets = s->hdr->next_ticket.load();
    return SVP_OK;
}

svp_status svp_ipc_shutdown(svp_ipc_server* hs) {
    if (!hs) {
        set_error("null server");
        return SVP_E_INVAL;
    }
    IpcServer* s = reinterpret_cast<IpcServer*>(hs);
    s->hdr->alive.store(0, std::memory_order_release);
    s->stop.store(true, std::memory_order_release);
    if (s->th.joinable()) s->th.join();
    // the arena must not be unregistered while svp jobs can still read it
    svp_flush(reinterpret_cast<svp_ctx*>(s->c));
    if (s->registered) executor_unregister_host(s->c->exec, s->arena);
    munmap(s->base, s->total);
    close(s->fd);
    shm_unlink((std::string("/") + s->name).c_str());
    delete s;
    return SVP_OK;
}

svp_status svp_ipc_connect(const char* name, svp_ipc_client** out) {
    if (!name || !out) {
        set_error("svp_ipc_connect: bad arguments");
        return SVP_E_INVAL;
    }
    *out = nullptr;
    IpcClient* c = new IpcClient();
    svp_status st = map_segment(name, false, 0, &c->fd, &c->base);
    if (st) {
        delete c;
        return st;
    }
    struct stat stt;
    fstat(c->fd, &stt);
    c->total = (uint64_t)stt.st_size;
    c->hdr = reinterpret_cast<IpcHeader*>(c->base);
    if (c->hdr->magic != kIpcMagic || c->hdr->total_bytes != c->total) {
        set_error("svp_ipc_connect: not an svp IPC segment (or not initialised yet)");
        munmap(c->base, c->total);
        close(c->fd);
        delete c;
        return SVP_E_INVAL;
    }
    c->slots = reinterpret_cast<IpcSlot*>(c->base + c->hdr->slots_off);
    c->arena = c->base + c->hdr->arena_off;
    *out = reinterpret_cast<svp_ipc_client*>(c);
    return SVP_OK;
}

svp_status svp_ipc_disconnect(svp_ipc_client* hc) {
    if (!hc) {
        set_error("null client");
        return SVP_E_INVAL;
    }
    IpcClient* c = reinterpret_cast<IpcClient*>(hc);
    munmap(c->base, c->total);
    close(c->fd);
    delete c;
    return SVP_OK;
}

svp_status svp_ipc_alloc(svp_ipc_client* hc, uint64_t bytes, uint64_t* offset_out, void** ptr_out) {
    if (!hc || !offset_out) {
        set_error("svp_ipc_alloc: bad arguments");
        return SVP_E_INVAL;
    }
    IpcClient* c = reinterpret_cast<IpcClient*>(hc);
    const uint64_t sz = align_up64(bytes ? bytes : 1, 256);
    const uint64_t off = c->hdr->arena_head.fetch_add(sz);
    if (off + sz > c->hdr->arena_bytes) {
        set_error("svp_ipc_alloc: shared arena exhausted");
        return SVP_E_NOMEM;
    }
    *offset_out = off;
    if (ptr_out) *ptr_out = c->arena + off;
    return SVP_OK;
}

svp_status svp_ipc_submit(svp_ipc_client* hc, int32_t vp, int32_t kernel, const void* args, size_t args_bytes,
                          const svp_ipc_buf* bufs, int32_t nbufs, uint64_t* ticket_out) {
    if (!hc || (!args && args_bytes) || args_bytes > SVP_MAX_ARGS || nbufs < 0 || nbufs > SVP_MAX_BUFS ||
        (!bufs && nbufs)) {
        set_error("svp_ipc_submit: bad arguments");
        return SVP_E_INVAL;
    }
    IpcClient* c = reinterpret_cast<IpcClient*>(hc);
    if (!c->hdr->alive.load(std::memory_order_acquire)) {
        set_error("svp_ipc_submit: server is gone");
        return SVP_E_STATE;
    }
    const uint64_t n = c->hdr->nslots;
    const uint64_t t = c->hdr->next_ticket.fetch_add(1);
    IpcSlot& sl = c->slots[t % n];
    for (int spins = 0;; ++spins) {
        if (sl.ticket.load(std::memory_order_acquire) == t && sl.state.load(std::memory_order_acquire) == SLOT_FREE)
            break;
        if (!c->hdr->alive.load(std::memory_order_acquire)) {
            set_error("svp_ipc_submit: server is gone");
            return SVP_E_STATE;
        }
        pause_briefly(spins);
    }
    sl.vp = vp;
    sl.kernel = kernel;
    sl.nbufs = nbufs;
    sl.args_bytes = (uint32_t)args_bytes;
    if (args_bytes) memcpy(sl.args, args, args_bytes);
    for (int b = 0; b < nbufs; ++b) {
        sl.bufs[b].off = bufs[b].offset;
        sl.bufs[b].bytes = bufs[b].bytes;
        sl.bufs[b].dir = bufs[b].dir;
    }
    sl.status = SVP_OK;
    sl.state.store(SLOT_SUBMITTED, std::memory_order_release);
    if (ticket_out) *ticket_out = t;
    return SVP_OK;
}

svp_status svp_ipc_wait(svp_ipc_client* hc, uint64_t ticket, int32_t timeout_ms) {
    if (!hc) {
        set_error("null client");
        return SVP_E_INVAL;
    }
    IpcClient* c = reinterpret_cast<IpcClient*>(hc);
    const uint64_t n = c->hdr->nslots;
    IpcSlot& sl = c->slots[ticket % n];
    auto deadline = std::chrono::steady_clock::now() + std::chrono::milliseconds(timeout_ms > 0 ? timeout_ms : 0);
    for (int spins = 0;; ++spins) {
        if (sl.ticket.load(std::memory_order_acquire) != ticket) {
            set_error("svp_ipc_wait: ticket not in flight (already waited?)");
            return SVP_E_INVAL;
        }
        if (sl.state.load(std::memory_order_acquire) == SLOT_DONE) break;
        if (!c->hdr->alive.load(std::memory_order_acquire)) {
            set_error("svp_ipc_wait: server is gone");
            return SVP_E_STATE;
        }
        if (timeout_ms > 0 && std::chrono::steady_clock::now() > deadline) {
            set_error("svp_ipc_wait: timed out");
            return SVP_E_TIMEOUT;
        }
        pause_briefly(spins);
    }
    const svp_status st = sl.status;
    sl.ticket.store(ticket + n, std::memory_order_relaxed);
    sl.state.store(SLOT_FREE, std::memory_order_release);  // recycle for ticket + n
    if (st) set_error("svp_ipc_wait: the job failed on the server");
    return st;
}

svp_status svp_kernel_lookup(const char* name, int32_t* id_out) {
    const KernelDesc* d = kernel_by_name(name);
    if (!d || !id_out) {
        set_error("svp_kernel_lookup: unknown kernel");
        return SVP_E_NOKERNEL;
    }
    *id_out = d->id;
    return SVP_OK;
}

}  // extern "C"
