// ipc.cpp -- cross-process zero-copy handoff of GPU objects.
//
// PAPER.md L167 (1): GROUTER "maps the address into the address space of
// function via CUDA IPC"; L269: data is allocated "from the local pool and
// mapped into the address space of functions using CUDA IPC"; L394: only
// pre-mapped storage is exposed to functions, and every access is
// authenticated.
//
// Isolation (R52).  An exported object lives in its OWN CUDA VMM
// allocation ("dedicated", exactly charge(n) bytes, POSIX-FD exportable):
// the first export of an object that still sits in a shared pool segment
// moves its bytes there once (one same-GPU copy) and frees the pool pages;
// later exports of the object reuse it.  An importer can therefore map the
// object's pages and nothing else.  The exporting context serves a dedicated
// allocation's file descriptor over an abstract Unix socket
// ("\0grouter.<pid>.<ctx_id>", SCM_RIGHTS) only:
//   * to a peer of the same uid (or root), checked with SO_PEERCRED, and
//   * for a LIVE export whose 128-bit random nonce, carried in the
//     descriptor, matches (the descriptor is the capability).
// A dedicated allocation never returns to the pool: when the exporter frees
// the object it unmaps its own view and releases its handle, and the physical
// pages stay alive exactly as long as an importer maps them (VMM reference
// counting) -- no page an importer still maps is ever reused for other data.
#include <sys/socket.h>
#include <sys/time.h>
#include <sys/un.h>
#include <unistd.h>

#include <atomic>
#include <cerrno>
#include <cstring>
#include <random>

#include "ctx.h"

namespace gr {

static std::atomic<uint32_t> g_ctx_ids{1};
static constexpr uint32_t kReqMagic = 0x47524958u;  // "GRIX"

static void sock_name(sockaddr_un &a, socklen_t &len, int pid, uint32_t ctx_id) {
  std::memset(&a, 0, sizeof(a));
  a.sun_family = AF_UNIX;
  std::string nm = "grouter." + std::to_string(pid) + "." + std::to_string(ctx_id);
  a.sun_path[0] = 0;  // abstract namespace
  std::memcpy(a.sun_path + 1, nm.data(), nm.size());
  len = (socklen_t)(offsetof(sockaddr_un, sun_path) + 1 + nm.size());
}

struct Req {
  uint32_t magic, pad;
  uint64_t export_id;
  uint64_t nonce[2];
};
struct Rsp {
  uint32_t ok, pad;
  uint64_t size;
};

// A peer that connects and then stalls must not hold the serving thread (or
// grouter_finalize, which joins it) -- nor an importer wait forever on a
// stalled exporter: every accepted / connecting socket gets I/O timeouts.
static void set_timeouts(int fd, int ms) {
  timeval tv{ms / 1000, (ms % 1000) * 1000};
  (void)::setsockopt(fd, SOL_SOCKET, SO_RCVTIMEO, &tv, sizeof(tv));
  (void)::setsockopt(fd, SOL_SOCKET, SO_SNDTIMEO, &tv, sizeof(tv));
}

static bool read_full(int fd, void *p, size_t n) {
  uint8_t *b = (uint8_t *)p;
  while (n) {
    ssize_t r = ::read(fd, b, n);
    if (r <= 0) return false;
    b += r;
    n -= (size_t)r;
  }
  return true;
}

static std::vector<CUmemAccessDesc> access_all(grouter_ctx *c) {
  std::vector<CUmemAccessDesc> ad;
  for (auto &kv : c->phys) {
    CUmemAccessDesc x = {};
    x.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    x.location.id = kv.first;
    x.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    ad.push_back(x);
  }
  return ad;
}

static void ded_release(Dedicated &d) {
  if (d.fd >= 0) ::close(d.fd);
  d.fd = -1;
  if (d.va) {
    drv().memUnmap(d.va, d.size);
    drv().memAddressFree(d.va, d.size);
    d.va = 0;
  }
  if (d.h) drv().memRelease(d.h);
  d.h = 0;
}

// Moves a sealed pool object into its own exportable VMM allocation (once).
// Caller holds c->mu; the object's bytes are in place (o.ready waited).
void ipc_dedicate(grouter_ctx *c, Obj &o) {
  const uint64_t len = charge(o.n);
  if (!len || c->dedicated.count((uint64_t)(uintptr_t)o.ptr)) return;
  LogicalDev &D = c->dev[o.loc];
  DeviceGuard g(D.phys);
  Dedicated d;
  d.logical = o.loc;
  d.phys = D.phys;
  d.size = len;
  CUmemAllocationProp prop = {};
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = D.phys;
  prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  if (drv().memCreate(&d.h, len, &prop, 0) != CUDA_SUCCESS) throw Error(GROUTER_ENOMEM, "export: cuMemCreate failed");
  try {
    GR_CU(drv().memAddressReserve(&d.va, len, kPage, 0, 0));
    GR_CU(drv().memMap(d.va, len, 0, d.h, 0));
    const std::vector<CUmemAccessDesc> ad = access_all(c);
    GR_CU(drv().memSetAccess(d.va, len, ad.data(), ad.size()));
    // one same-GPU copy on the copy server's stream (ordered after its
    // earlier rounds); export blocks until the bytes are in place anyway
    GR_CUDA(cudaMemcpyAsync((void *)d.va, o.ptr, o.n, cudaMemcpyDeviceToDevice, D.copy.stream));
    EventRef e = record(c, D.copy.stream, D.phys);
    GR_CUDA(cudaEventSynchronize(e->ev));
  } catch (...) {
    ded_release(d);
    throw;
  }
  Fences old = std::move(o.readers);
  for (auto &w : o.ready) old.push_back(w);
  dev_free(c, o.loc, o.ptr, len, std::move(old));  // the shared pool pages go back
  o.ready.clear();
  o.readers.clear();
  o.ptr = (uint8_t *)(uintptr_t)d.va;
  c->dedicated.emplace(d.va, d);
}

// Registers a live export of the dedicated allocation at `va`: returns its id
// and a fresh 128-bit random nonce.  Caller holds c->mu.
uint64_t ipc_export_record(grouter_ctx *c, uint64_t va, uint64_t nonce[2]) {
  Dedicated &d = c->dedicated.at(va);
  if (d.fd < 0) GR_CU(drv().memExportToShareableHandle(&d.fd, d.h, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0));
  static thread_local std::random_device rd;  // /dev/urandom (getrandom) on Linux
  for (int i = 0; i < 2; ++i) nonce[i] = ((uint64_t)rd() << 32) ^ (uint64_t)rd();
  const uint64_t id = c->next_export_id++;
  c->exports[id] = ExportRec{{nonce[0], nonce[1]}, va};
  d.export_ids.push_back(id);
  return id;
}

// dev_free for a dedicated allocation: its exports end now (no new imports),
// its own mapping goes once the object's GPU work is done (ded_sweep).
// Returns false if p is not a dedicated allocation.  Caller holds c->mu.
bool ded_free(grouter_ctx *c, uint8_t *p, Fences &&f) {
  auto it = c->dedicated.find((uint64_t)(uintptr_t)p);
  if (it == c->dedicated.end()) return false;
  for (uint64_t id : it->second.export_ids) c->exports.erase(id);
  it->second.export_ids.clear();
  c->ded_retire.push_back({it->second, std::move(f)});
  c->dedicated.erase(it);
  return true;
}

// Unmaps and releases retired dedicated allocations whose fences completed.
// The driver calls run WITHOUT the context lock when `lk` is given (an unmap
// drains the GPU; the pool trim does the same).
void ded_sweep(grouter_ctx *c, std::unique_lock<std::mutex> *lk, bool wait) {
  std::vector<Dedicated> done;
  size_t w = 0;
  for (size_t i = 0; i < c->ded_retire.size(); ++i) {
    DedRetire &r = c->ded_retire[i];
    bool ok = true;
    if (wait) host_wait(r.f);
    else
      for (auto &x : r.f) ok &= x.done();
    if (ok) {
      done.push_back(r.d);
    } else {
      if (w != i) c->ded_retire[w] = std::move(c->ded_retire[i]);
      ++w;
    }
  }
  c->ded_retire.resize(w);
  if (done.empty()) return;
  if (lk) lk->unlock();
  for (auto &d : done) {
    DeviceGuard g(d.phys);
    ded_release(d);
  }
  if (lk) lk->lock();
}

static void serve(grouter_ctx *c) {
  for (;;) {
    int cfd = ::accept(c->ipc_listen, nullptr, nullptr);
    if (cfd < 0) {
      if (errno == EINTR) continue;
      return;  // listening socket closed: shutting down
    }
    set_timeouts(cfd, 1000);
    Req rq;
    Rsp rsp{0, 0, 0};
    int fd = -1;
    ucred cr{};
    socklen_t crl = sizeof(cr);
    const bool peer_ok = ::getsockopt(cfd, SOL_SOCKET, SO_PEERCRED, &cr, &crl) == 0 &&
                         (cr.uid == ::getuid() || cr.uid == 0);
    if (peer_ok && read_full(cfd, &rq, sizeof(rq)) && rq.magic == kReqMagic) {
      std::lock_guard<std::mutex> g(c->mu);
      auto it = c->exports.find(rq.export_id);
      if (it != c->exports.end()) {
        const ExportRec &e = it->second;
        const uint64_t diff = (e.nonce[0] ^ rq.nonce[0]) | (e.nonce[1] ^ rq.nonce[1]);
        auto d = c->dedicated.find(e.va);
        if (diff == 0 && d != c->dedicated.end() && d->second.fd >= 0) {
          rsp.ok = 1;
          rsp.size = d->second.size;
          fd = ::dup(d->second.fd);  // sent while the allocation may be retired concurrently
          if (fd < 0) rsp.ok = 0;
        }
      }
    }
    iovec iov{&rsp, sizeof(rsp)};
    msghdr m{};
    m.msg_iov = &iov;
    m.msg_iovlen = 1;
    char cbuf[CMSG_SPACE(sizeof(int))];
    if (rsp.ok) {
      m.msg_control = cbuf;
      m.msg_controllen = CMSG_SPACE(sizeof(int));
      cmsghdr *cm = CMSG_FIRSTHDR(&m);
      cm->cmsg_level = SOL_SOCKET;
      cm->cmsg_type = SCM_RIGHTS;
      cm->cmsg_len = CMSG_LEN(sizeof(int));
      std::memcpy(CMSG_DATA(cm), &fd, sizeof(int));
    }
    (void)::sendmsg(cfd, &m, MSG_NOSIGNAL);
    if (fd >= 0) ::close(fd);
    ::close(cfd);
  }
}

void ipc_serve_start(grouter_ctx *c) {
  if (c->ipc_listen >= 0) return;
  if (!c->ctx_id) c->ctx_id = g_ctx_ids.fetch_add(1);
  int fd = ::socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
  if (fd < 0) throw Error(GROUTER_ECUDA, "ipc: socket() failed");
  sockaddr_un a;
  socklen_t len;
  sock_name(a, len, (int)::getpid(), c->ctx_id);
  if (::bind(fd, (sockaddr *)&a, len) != 0 || ::listen(fd, 64) != 0) {
    ::close(fd);
    throw Error(GROUTER_ECUDA, "ipc: bind/listen failed");
  }
  c->ipc_listen = fd;
  c->ipc_thread = std::thread(serve, c);
}

// Stops serving; the context's remaining dedicated allocations are released
// by the caller's teardown (ipc_release_all).
void ipc_shutdown(grouter_ctx *c) {
  if (c->ipc_listen >= 0) {
    ::shutdown(c->ipc_listen, SHUT_RDWR);
    ::close(c->ipc_listen);
    c->ipc_listen = -1;
  }
  if (c->ipc_thread.joinable()) c->ipc_thread.join();
  c->exports.clear();
}

void ipc_release_all(grouter_ctx *c) {
  for (auto &kv : c->dedicated) {
    DeviceGuard g(kv.second.phys);
    ded_release(kv.second);
  }
  c->dedicated.clear();
  for (auto &r : c->ded_retire) {
    DeviceGuard g(r.d.phys);
    ded_release(r.d);
  }
  c->ded_retire.clear();
}

std::shared_ptr<RemoteMap> ipc_map(grouter_ctx *c, const grouter_ipc_desc &d, int local_phys) {
  int s = ::socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
  if (s < 0) throw Error(GROUTER_ECUDA, "ipc: socket() failed");
  sockaddr_un a;
  socklen_t len;
  sock_name(a, len, d.pid, d.ctx_id);
  set_timeouts(s, 10000);
  if (::connect(s, (sockaddr *)&a, len) != 0) {
    ::close(s);
    throw Error(GROUTER_EINVAL, "ipc: exporter not reachable (process gone or other namespace)");
  }
  Req rq{};
  rq.magic = kReqMagic;
  rq.export_id = d.export_id;
  rq.nonce[0] = d.nonce[0];
  rq.nonce[1] = d.nonce[1];
  if (::write(s, &rq, sizeof(rq)) != (ssize_t)sizeof(rq)) {
    ::close(s);
    throw Error(GROUTER_ECUDA, "ipc: request failed");
  }
  Rsp rsp{};
  iovec iov{&rsp, sizeof(rsp)};
  msghdr m{};
  m.msg_iov = &iov;
  m.msg_iovlen = 1;
  char cbuf[CMSG_SPACE(sizeof(int))];
  m.msg_control = cbuf;
  m.msg_controllen = sizeof(cbuf);
  ssize_t r = ::recvmsg(s, &m, MSG_WAITALL);
  ::close(s);
  cmsghdr *cm = (r == (ssize_t)sizeof(rsp) && rsp.ok) ? CMSG_FIRSTHDR(&m) : nullptr;
  if (!cm || cm->cmsg_type != SCM_RIGHTS)
    throw Error(GROUTER_ENOENT, "ipc: export refused (freed object, wrong nonce, or another user)");
  int fd = -1;
  std::memcpy(&fd, CMSG_DATA(cm), sizeof(int));
  if (rsp.size != d.alloc_bytes || rsp.size < d.n) {
    ::close(fd);
    throw Error(GROUTER_EINVAL, "ipc: exporter's allocation does not match the descriptor");
  }
  auto map = std::make_shared<RemoteMap>();
  map->phys = local_phys;
  try {
    CUmemGenericAllocationHandle h;
    GR_CU(drv().memImportFromShareableHandle(&h, (void *)(uintptr_t)fd, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR));
    map->handles.push_back(h);
    map->sizes.push_back(rsp.size);
    GR_CU(drv().memAddressReserve(&map->va, rsp.size, kPage, 0, 0));
    map->size = rsp.size;
    GR_CU(drv().memMap(map->va, rsp.size, 0, h, 0));
    const std::vector<CUmemAccessDesc> ad = access_all(c);
    GR_CU(drv().memSetAccess(map->va, rsp.size, ad.data(), ad.size()));
  } catch (...) {
    ::close(fd);
    ipc_unmap(*map);
    throw;
  }
  ::close(fd);
  return map;
}

void ipc_unmap(RemoteMap &m) {
  if (m.va) {
    uint64_t off = 0;
    for (size_t i = 0; i < m.sizes.size() && off < m.size; ++i) {
      drv().memUnmap(m.va + off, m.sizes[i]);
      off += m.sizes[i];
    }
    drv().memAddressFree(m.va, m.size);
    m.va = 0;
  }
  for (auto h : m.handles) drv().memRelease(h);
  m.handles.clear();
}

}  // namespace gr
