// ipc.cpp -- cross-process zero-copy handoff of pool pages.
//
// PAPER.md L167 (1): GROUTER "maps the address into the address space of
// function via CUDA IPC"; L269: data is allocated "from the local pool and
// mapped into the address space of functions using CUDA IPC"; L394: only
// pre-mapped storage is exposed, authenticated by workflow.
//
// Pool segments are CUDA VMM allocations created with
// CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR.  An exporting context serves the
// file descriptors of requested segments over an abstract Unix socket
// ("\0grouter.<pid>.<ctx_id>", SCM_RIGHTS); the importer maps them into a
// fresh virtual range with access for its GPU.  Same GPU: the importer's
// pointer aliases the exporter's bytes (zero copy).  Other GPU: the mapping
// is a peer mapping that the SM copy kernel reads over NVLink.
#include <sys/socket.h>
#include <sys/un.h>
#include <unistd.h>

#include <atomic>
#include <cerrno>
#include <cstring>

#include "ctx.h"

namespace gr {

static std::atomic<uint32_t> g_ctx_ids{1};

static void sock_name(sockaddr_un &a, socklen_t &len, int pid, uint32_t ctx_id) {
  std::memset(&a, 0, sizeof(a));
  a.sun_family = AF_UNIX;
  std::string nm = "grouter." + std::to_string(pid) + "." + std::to_string(ctx_id);
  a.sun_path[0] = 0;  // abstract namespace
  std::memcpy(a.sun_path + 1, nm.data(), nm.size());
  len = (socklen_t)(offsetof(sockaddr_un, sun_path) + 1 + nm.size());
}

struct Req {
  uint32_t magic, n;
  int32_t logical;
  uint32_t pad;
  uint64_t seg_off[GROUTER_IPC_MAX_SEGS];
};

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

// Returns the exported fd of a pool segment (cached); caller holds c->mu.
static int segment_fd(grouter_ctx *c, int logical, uint64_t seg_off, uint64_t *size) {
  DevicePool &P = c->dev[logical].pool;
  for (auto &s : P.segs) {
    if (s.off != seg_off) continue;
    *size = s.size;
    auto key = std::make_pair(logical, seg_off);
    auto it = c->exported_fds.find(key);
    if (it != c->exported_fds.end()) return it->second;
    int fd = -1;
    GR_CU(drv().memExportToShareableHandle(&fd, s.h, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0));
    c->exported_fds[key] = fd;
    return fd;
  }
  return -1;
}

static void serve(grouter_ctx *c) {
  for (;;) {
    int cfd = ::accept(c->ipc_listen, nullptr, nullptr);
    if (cfd < 0) {
      if (errno == EINTR) continue;
      return;  // listening socket closed: shutting down
    }
    Req rq;
    if (read_full(cfd, &rq, sizeof(rq)) && rq.magic == 0x47524950u && rq.n <= GROUTER_IPC_MAX_SEGS) {
      int fds[GROUTER_IPC_MAX_SEGS];
      uint64_t sizes[GROUTER_IPC_MAX_SEGS] = {};
      uint32_t ok = 1;
      {
        std::lock_guard<std::mutex> g(c->mu);
        try {
          if (rq.logical < 0 || rq.logical >= (int)c->dev.size()) ok = 0;
          for (uint32_t i = 0; ok && i < rq.n; ++i) {
            fds[i] = segment_fd(c, rq.logical, rq.seg_off[i], &sizes[i]);
            if (fds[i] < 0) ok = 0;
          }
        } catch (...) {
          ok = 0;
        }
      }
      struct {
        uint32_t ok, n;
        uint64_t sizes[GROUTER_IPC_MAX_SEGS];
      } rsp{ok, ok ? rq.n : 0, {}};
      std::memcpy(rsp.sizes, sizes, sizeof(sizes));
      iovec iov{&rsp, sizeof(rsp)};
      msghdr m{};
      m.msg_iov = &iov;
      m.msg_iovlen = 1;
      char cbuf[CMSG_SPACE(sizeof(int) * GROUTER_IPC_MAX_SEGS)];
      if (ok && rq.n) {
        m.msg_control = cbuf;
        m.msg_controllen = CMSG_SPACE(sizeof(int) * rq.n);
        cmsghdr *cm = CMSG_FIRSTHDR(&m);
        cm->cmsg_level = SOL_SOCKET;
        cm->cmsg_type = SCM_RIGHTS;
        cm->cmsg_len = CMSG_LEN(sizeof(int) * rq.n);
        std::memcpy(CMSG_DATA(cm), fds, sizeof(int) * rq.n);
      }
      (void)::sendmsg(cfd, &m, 0);
    }
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

void ipc_shutdown(grouter_ctx *c) {
  if (c->ipc_listen >= 0) {
    ::shutdown(c->ipc_listen, SHUT_RDWR);
    ::close(c->ipc_listen);
    c->ipc_listen = -1;
  }
  if (c->ipc_thread.joinable()) c->ipc_thread.join();
  for (auto &kv : c->exported_fds) ::close(kv.second);
  c->exported_fds.clear();
}

std::shared_ptr<RemoteMap> ipc_map(grouter_ctx *c, const grouter_ipc_desc &d, int local_phys) {
  int s = ::socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
  if (s < 0) throw Error(GROUTER_ECUDA, "ipc: socket() failed");
  sockaddr_un a;
  socklen_t len;
  sock_name(a, len, d.pid, d.ctx_id);
  if (::connect(s, (sockaddr *)&a, len) != 0) {
    ::close(s);
    throw Error(GROUTER_EINVAL, "ipc: exporter not reachable (process gone or other namespace)");
  }
  Req rq{};
  rq.magic = 0x47524950u;
  rq.n = d.n_segs;
  rq.logical = d.logical;
  for (uint32_t i = 0; i < d.n_segs; ++i) rq.seg_off[i] = d.seg_off[i];
  if (::write(s, &rq, sizeof(rq)) != (ssize_t)sizeof(rq)) {
    ::close(s);
    throw Error(GROUTER_ECUDA, "ipc: request failed");
  }
  struct {
    uint32_t ok, n;
    uint64_t sizes[GROUTER_IPC_MAX_SEGS];
  } rsp{};
  iovec iov{&rsp, sizeof(rsp)};
  msghdr m{};
  m.msg_iov = &iov;
  m.msg_iovlen = 1;
  char cbuf[CMSG_SPACE(sizeof(int) * GROUTER_IPC_MAX_SEGS)];
  m.msg_control = cbuf;
  m.msg_controllen = sizeof(cbuf);
  ssize_t r = ::recvmsg(s, &m, MSG_WAITALL);
  ::close(s);
  if (r != (ssize_t)sizeof(rsp) || !rsp.ok || rsp.n != d.n_segs)
    throw Error(GROUTER_EINVAL, "ipc: exporter refused the segments");
  int fds[GROUTER_IPC_MAX_SEGS];
  cmsghdr *cm = CMSG_FIRSTHDR(&m);
  if (!cm || cm->cmsg_type != SCM_RIGHTS) throw Error(GROUTER_ECUDA, "ipc: no descriptors received");
  std::memcpy(fds, CMSG_DATA(cm), sizeof(int) * rsp.n);
  auto map = std::make_shared<RemoteMap>();
  map->phys = local_phys;
  uint64_t total = 0;
  for (uint32_t i = 0; i < rsp.n; ++i) total += rsp.sizes[i];
  try {
    for (uint32_t i = 0; i < rsp.n; ++i) {
      CUmemGenericAllocationHandle h;
      GR_CU(drv().memImportFromShareableHandle(&h, (void *)(uintptr_t)fds[i],
                                               CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR));
      map->handles.push_back(h);
      map->sizes.push_back(rsp.sizes[i]);
    }
    GR_CU(drv().memAddressReserve(&map->va, total, kPage, 0, 0));
    map->size = total;
    uint64_t off = 0;
    for (size_t i = 0; i < map->handles.size(); ++i) {
      GR_CU(drv().memMap(map->va + off, map->sizes[i], 0, map->handles[i], 0));
      off += map->sizes[i];
    }
    std::vector<CUmemAccessDesc> ad;
    for (auto &kv : c->phys) {
      CUmemAccessDesc x = {};
      x.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
      x.location.id = kv.first;
      x.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
      ad.push_back(x);
    }
    GR_CU(drv().memSetAccess(map->va, total, ad.data(), ad.size()));
  } catch (...) {
    for (uint32_t i = 0; i < rsp.n; ++i) ::close(fds[i]);
    ipc_unmap(*map);
    throw;
  }
  for (uint32_t i = 0; i < rsp.n; ++i) ::close(fds[i]);
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
