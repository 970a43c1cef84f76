// File-descriptor exchange between the ranks of one node (mpress_share_fds).
//
// cuMem pools are exported as POSIX file descriptors
// (CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR).  A descriptor only means
// something inside the process that owns it, so it cannot travel through the
// torch process group; it is passed with SCM_RIGHTS over a Unix-domain
// socket, which makes the kernel install a duplicate in the receiver.
//
// Rendezvous (three all-gathers through the caller's exchange callback):
//   1. every rank contributes {pid, nonce, want[world]}; rank 0's nonce names
//      the job, so concurrent jobs on one node never collide;
//   2. after every rank listens on "\0mpress.<nonce>.<rank>" (abstract
//      namespace: no filesystem entry to clean up);
//   3. after every descriptor has been delivered (then listeners close).
// Rank p serves its fd to each rank r with want_r[p] != 0 from a helper
// thread while the main thread fetches the fds it wants itself; a connection
// is served only when SO_PEERCRED names one of those ranks (pid and uid).
#include <poll.h>
#include <sys/socket.h>
#include <sys/un.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <cerrno>
#include <cstring>
#include <random>
#include <string>
#include <thread>
#include <vector>

#include "common.h"

namespace mpress {
namespace {

constexpr int kTimeoutMs = 120000;

struct Hello {
  int32_t pid;
  int32_t rank;
  uint64_t nonce;
};

socklen_t make_addr(uint64_t nonce, int rank, sockaddr_un* a) {
  memset(a, 0, sizeof *a);
  a->sun_family = AF_UNIX;
  char name[96];
  int n = snprintf(name, sizeof name, "mpress.%016llx.%d", (unsigned long long)nonce, rank);
  a->sun_path[0] = '\0';  // abstract namespace
  memcpy(a->sun_path + 1, name, n);
  return (socklen_t)(offsetof(sockaddr_un, sun_path) + 1 + n);
}

int send_fd(int sock, int fd, int32_t rank) {
  msghdr msg{};
  iovec iov{&rank, sizeof rank};
  msg.msg_iov = &iov;
  msg.msg_iovlen = 1;
  alignas(cmsghdr) char cbuf[CMSG_SPACE(sizeof(int))];
  memset(cbuf, 0, sizeof cbuf);
  msg.msg_control = cbuf;
  msg.msg_controllen = sizeof cbuf;
  cmsghdr* c = CMSG_FIRSTHDR(&msg);
  c->cmsg_level = SOL_SOCKET;
  c->cmsg_type = SCM_RIGHTS;
  c->cmsg_len = CMSG_LEN(sizeof(int));
  memcpy(CMSG_DATA(c), &fd, sizeof fd);
  ssize_t r;
  do { r = sendmsg(sock, &msg, MSG_NOSIGNAL); } while (r < 0 && errno == EINTR);
  return r == (ssize_t)sizeof rank ? 0 : -1;
}

int recv_fd(int sock, int32_t* rank_out) {
  msghdr msg{};
  int32_t rank = -1;
  iovec iov{&rank, sizeof rank};
  msg.msg_iov = &iov;
  msg.msg_iovlen = 1;
  alignas(cmsghdr) char cbuf[CMSG_SPACE(sizeof(int))];
  msg.msg_control = cbuf;
  msg.msg_controllen = sizeof cbuf;
  ssize_t r;
  do { r = recvmsg(sock, &msg, MSG_CMSG_CLOEXEC); } while (r < 0 && errno == EINTR);
  if (r != (ssize_t)sizeof rank) return -1;
  cmsghdr* c = CMSG_FIRSTHDR(&msg);
  if (!c || c->cmsg_level != SOL_SOCKET || c->cmsg_type != SCM_RIGHTS) return -1;
  int fd;
  memcpy(&fd, CMSG_DATA(c), sizeof fd);
  *rank_out = rank;
  return fd;
}

void set_timeouts(int sock) {
  timeval tv{kTimeoutMs / 1000, 0};
  setsockopt(sock, SOL_SOCKET, SO_RCVTIMEO, &tv, sizeof tv);
  setsockopt(sock, SOL_SOCKET, SO_SNDTIMEO, &tv, sizeof tv);
}

}  // namespace
}  // namespace mpress

using namespace mpress;

extern "C" int mpress_share_fds(int world, int rank, int my_fd, const int32_t* want,
                                mpress_exchange_fn exchange, void* exchange_user,
                                int32_t* fds_out) {
  if (world < 1 || rank < 0 || rank >= world || !want || !exchange || !fds_out)
    return fail(MPRESS_ERR_ARG, "mpress_share_fds: bad argument");
  for (int p = 0; p < world; ++p) fds_out[p] = -1;

  // ---- 1. hello: pid, nonce, want vector --------------------------------
  const size_t rec = sizeof(Hello) + (size_t)world;
  std::vector<uint8_t> mine(rec), all(rec * world);
  Hello h{(int32_t)getpid(), rank, 0};
  {
    std::random_device rd;
    h.nonce = ((uint64_t)rd() << 32) ^ rd() ^ ((uint64_t)getpid() << 16) ^ (uint64_t)time(nullptr);
  }
  memcpy(mine.data(), &h, sizeof h);
  for (int p = 0; p < world; ++p) mine[sizeof(Hello) + p] = (want[p] && p != rank) ? 1 : 0;
  if (exchange(exchange_user, mine.data(), rec, all.data()) != 0)
    return fail(MPRESS_ERR_SYS, "mpress_share_fds: exchange #1 failed");
  Hello h0;
  memcpy(&h0, all.data(), sizeof h0);
  const uint64_t nonce = h0.nonce;
  int incoming = 0;
  for (int r = 0; r < world; ++r)
    if (all[(size_t)r * rec + sizeof(Hello) + rank]) ++incoming;
  if (incoming > 0 && my_fd < 0)
    return fail(MPRESS_ERR_ARG, "mpress_share_fds: rank %d has no fd to offer", rank);

  // ---- 2. listen, barrier ------------------------------------------------
  int lsock = -1;
  int rc_listen = 0;
  if (incoming > 0) {
    lsock = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
    sockaddr_un a;
    socklen_t alen = make_addr(nonce, rank, &a);
    if (lsock < 0 || bind(lsock, (sockaddr*)&a, alen) != 0 || listen(lsock, world) != 0)
      rc_listen = errno ? errno : -1;
  }
  int32_t ok_mine = rc_listen == 0 ? 1 : 0;
  std::vector<int32_t> ok_all(world);
  if (exchange(exchange_user, &ok_mine, sizeof ok_mine, ok_all.data()) != 0) {
    if (lsock >= 0) close(lsock);
    return fail(MPRESS_ERR_SYS, "mpress_share_fds: exchange #2 failed");
  }
  for (int r = 0; r < world; ++r) {
    if (!ok_all[r]) {
      if (lsock >= 0) close(lsock);
      return fail(MPRESS_ERR_SYS, "mpress_share_fds: rank %d could not listen (%s)", r,
                  r == rank ? strerror(rc_listen) : "remote");
    }
  }

  // ---- serve my fd from a helper thread ----------------------------------
  std::atomic<int> serve_err{0};
  std::thread server;
  if (incoming > 0) {
    // The ranks allowed to fetch this fd: those whose want vector names this
    // rank.  The abstract socket name is visible to every local user
    // (/proc/net/unix), so a connection is served only if the kernel's
    // credentials of the peer (SO_PEERCRED) are one of those ranks' pid with
    // this process's uid; anything else is closed and not counted.
    std::vector<int32_t> allowed;
    for (int r = 0; r < world; ++r)
      if (r != rank && all[(size_t)r * rec + sizeof(Hello) + rank]) {
        Hello hr;
        memcpy(&hr, all.data() + (size_t)r * rec, sizeof hr);
        allowed.push_back(hr.pid);
      }
    server = std::thread([&, allowed]() mutable {
      timespec t0;
      clock_gettime(CLOCK_MONOTONIC, &t0);
      for (int i = 0; i < incoming;) {
        timespec t1;
        clock_gettime(CLOCK_MONOTONIC, &t1);
        const long left = kTimeoutMs - ((t1.tv_sec - t0.tv_sec) * 1000 + (t1.tv_nsec - t0.tv_nsec) / 1000000);
        pollfd pf{lsock, POLLIN, 0};
        if (left <= 0 || poll(&pf, 1, (int)left) <= 0) { serve_err = ETIMEDOUT; return; }
        int c = accept4(lsock, nullptr, nullptr, SOCK_CLOEXEC);
        if (c < 0) { serve_err = errno; return; }
        ucred cred{};
        socklen_t clen = sizeof cred;
        auto who = allowed.end();
        if (getsockopt(c, SOL_SOCKET, SO_PEERCRED, &cred, &clen) == 0 && cred.uid == getuid())
          who = std::find(allowed.begin(), allowed.end(), (int32_t)cred.pid);
        if (who == allowed.end()) {  // not one of this job's ranks (or already served)
          close(c);
          continue;
        }
        allowed.erase(who);
        ++i;
        set_timeouts(c);
        if (send_fd(c, my_fd, rank) != 0) serve_err = errno ? errno : EIO;
        // wait for the peer's 1-byte ack so the fd is received before we close
        char ack;
        if (recv(c, &ack, 1, 0) != 1 && !serve_err) serve_err = EIO;
        close(c);
        if (serve_err) return;
      }
    });
  }

  // ---- fetch the fds I want -------------------------------------------------
  int fetch_rc = MPRESS_OK;
  for (int p = 0; p < world && fetch_rc == MPRESS_OK; ++p) {
    if (p == rank || !want[p]) continue;
    sockaddr_un a;
    socklen_t alen = make_addr(nonce, p, &a);
    int tries = 0;
    int s = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
    while (s >= 0 && connect(s, (sockaddr*)&a, alen) != 0) {
      close(s);  // a failed connect leaves the socket unusable: start afresh
      s = -1;
      if (++tries > 2000) break;
      usleep(1000);
      s = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
    }
    if (s < 0 || tries > 2000) {
      fetch_rc = fail(MPRESS_ERR_SYS, "mpress_share_fds: connect to rank %d failed: %s", p, strerror(errno));
      if (s >= 0) close(s);
      break;
    }
    set_timeouts(s);
    int32_t from = -1;
    int fd = recv_fd(s, &from);
    if (fd < 0 || from != p) {
      fetch_rc = fail(MPRESS_ERR_SYS, "mpress_share_fds: no descriptor from rank %d", p);
    } else {
      fds_out[p] = fd;
      char ack = 1;
      (void)!send(s, &ack, 1, MSG_NOSIGNAL);
    }
    close(s);
  }
  if (server.joinable()) server.join();
  if (lsock >= 0) close(lsock);
  if (fetch_rc == MPRESS_OK && serve_err)
    fetch_rc = fail(MPRESS_ERR_SYS, "mpress_share_fds: serving rank %d failed: %s", rank, strerror(serve_err));

  // ---- 3. everyone done (listeners may now disappear) ----------------------
  int32_t done_mine = fetch_rc == MPRESS_OK ? 1 : 0;
  if (exchange(exchange_user, &done_mine, sizeof done_mine, ok_all.data()) != 0 && fetch_rc == MPRESS_OK)
    fetch_rc = fail(MPRESS_ERR_SYS, "mpress_share_fds: exchange #3 failed");
  if (fetch_rc == MPRESS_OK) {
    for (int r = 0; r < world; ++r)
      if (!ok_all[r]) { fetch_rc = fail(MPRESS_ERR_SYS, "mpress_share_fds: rank %d failed", r); break; }
  }
  if (fetch_rc != MPRESS_OK) {
    for (int p = 0; p < world; ++p)
      if (fds_out[p] >= 0) { close(fds_out[p]); fds_out[p] = -1; }
  }
  return fetch_rc;
}
