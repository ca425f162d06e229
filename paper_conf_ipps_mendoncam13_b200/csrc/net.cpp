// net.cpp — TCP transport of the master/slave protocol (see net.h).  Messages are
// fixed-size little-endian structs on a loopback socket (one node); the master's task
// table is the same sw_sched core the in-process driver uses.
#include "net.h"
#include <arpa/inet.h>
#include <netdb.h>
#include <netinet/in.h>
#include <netinet/tcp.h>
#include <sys/socket.h>
#include <unistd.h>
#include <chrono>
#include <cstring>
#include <stdexcept>
#include "sw_internal.h"
#include "../../include/sw.h"

namespace sw {

namespace {
enum Op : int32_t { kHello = 0, kRequest = 1, kReport = 2, kComplete = 3, kAbandon = 4,
                    kFinishedMap = 5, kDone = 6, kCounters = 7, kStart = 8, kRequestWait = 9 };
struct Msg {
  int32_t op, worker, unit, cap;
  double t, cells, sec;   // kRequestWait: sec = timeout
  uint64_t hash;          // kHello: the slave's plan hash
};
struct RepHdr {
  int32_t rc, nextra;
};

double now_s() {
  using namespace std::chrono;
  return duration<double>(steady_clock::now().time_since_epoch()).count();
}
bool send_all(int fd, const void *p, size_t n) {
  const char *c = static_cast<const char *>(p);
  while (n) {
    ssize_t k = ::send(fd, c, n, MSG_NOSIGNAL);
    if (k <= 0) return false;
    c += k; n -= (size_t)k;
  }
  return true;
}
bool recv_all(int fd, void *p, size_t n) {
  char *c = static_cast<char *>(p);
  while (n) {
    ssize_t k = ::recv(fd, c, n, 0);
    if (k <= 0) return false;
    c += k; n -= (size_t)k;
  }
  return true;
}
void nodelay(int fd) {
  int one = 1;
  setsockopt(fd, IPPROTO_TCP, TCP_NODELAY, &one, sizeof(one));
}
}  // namespace

MasterServer::~MasterServer() { stop(); }

void MasterServer::start(int port, int world, int32_t n_units, const int64_t *unit_cells,
                         int32_t policy, int32_t wa, int32_t omega, uint64_t plan_hash) {
  world_ = world;
  plan_hash_ = plan_hash;
  sched_ = sw_sched_create(world, n_units, unit_cells, policy, wa, omega);
  if (!sched_ && n_units > 0) throw Error(SW_EINVAL, "master: scheduler creation failed");
  listen_fd_ = ::socket(AF_INET, SOCK_STREAM, 0);
  if (listen_fd_ < 0) throw Error(SW_ENET, "master: socket() failed");
  int one = 1;
  setsockopt(listen_fd_, SOL_SOCKET, SO_REUSEADDR, &one, sizeof(one));
  sockaddr_in a{};
  a.sin_family = AF_INET;
  a.sin_addr.s_addr = htonl(INADDR_ANY);
  a.sin_port = htons((uint16_t)port);
  if (::bind(listen_fd_, (sockaddr *)&a, sizeof(a)) != 0 || ::listen(listen_fd_, 64) != 0) {
    ::close(listen_fd_);
    listen_fd_ = -1;
    throw Error(SW_ENET, "master: cannot bind/listen on port " + std::to_string(port));
  }
  // "the master process starts the execution and waits for the slaves to register" (P16)
  accept_thread_ = std::thread([this] {
    for (int k = 0; k < world_; k++) {
      int fd = ::accept(listen_fd_, nullptr, nullptr);
      if (fd < 0) break;
      nodelay(fd);
      std::lock_guard<std::mutex> g(mu_);
      conns_.emplace_back([this, fd] { serve(fd); });
    }
  });
}

void MasterServer::serve(int fd) {
  Msg m;
  std::vector<int32_t> buf;
  int32_t worker = -1;
  bool left = false;
  while (recv_all(fd, &m, sizeof(m))) {
    RepHdr h{0, 0};
    buf.clear();
    const double t = now_s();  // the master's clock
    switch (m.op) {
      case kHello:
        // a slave whose unit table differs from rank 0's would execute other (pack, group)
        // ranges under the same unit ids: refuse it
        if (m.hash != plan_hash_) { h.rc = -1; break; }
        worker = m.worker;
        registered_.fetch_add(1);
        break;
      case kRequest:
      case kRequestWait: {
        // "the master process starts the execution and waits for the slaves to register"
        // (P16 §IV): no task is handed out before every slave has registered
        if (registered_.load() < world_) {
          if (m.op == kRequestWait) std::this_thread::sleep_for(std::chrono::milliseconds(1));
          h.rc = 0;
          break;
        }
        buf.resize(std::max(1, m.cap));
        if (!sched_) h.rc = -1;
        else if (m.op == kRequest) h.rc = sw_sched_request(sched_, worker, t, buf.data(), m.cap);
        else h.rc = sw_sched_request_wait(sched_, worker, t, buf.data(), m.cap, m.sec);
        buf.resize(h.rc > 0 ? h.rc : 0);
        break;
      }
      case kReport: if (sched_) sw_sched_report(sched_, worker, t, m.cells, m.sec); break;
      case kComplete: h.rc = sched_ ? sw_sched_complete(sched_, worker, m.unit, t) : 1; break;
      case kAbandon: if (sched_) sw_sched_abandon(sched_, worker, m.unit, t); break;
      case kStart: h.rc = sched_ ? sw_sched_start(sched_, worker, m.unit, t) : 1; break;
      case kFinishedMap: {
        const int32_t n = m.cap;
        buf.assign((n + 31) / 32, 0);
        for (int32_t u = 0; u < n; u++)
          if (sched_ && sw_sched_is_finished(sched_, u)) buf[u / 32] |= (int32_t)(1u << (u % 32));
        break;
      }
      case kCounters:
        buf.assign(3, 0);
        if (sched_)
          for (int k = 0; k < 3; k++) buf[k] = (int32_t)sw_sched_counter(sched_, k == 2 ? 3 : k);
        break;
      case kDone: done_.fetch_add(1); left = true; break;
      default: break;
    }
    h.nextra = (int32_t)buf.size();
    if (!send_all(fd, &h, sizeof(h)) || (h.nextra && !send_all(fd, buf.data(), sizeof(int32_t) * buf.size())))
      break;
    if (m.op == kDone || (m.op == kHello && h.rc < 0)) break;
  }
  if (!left) {
    // the connection closed without DONE: the slave is gone; its unfinished tasks go back
    // to READY so the others can still finish the search (and stop() does not wait for it)
    if (sched_ && worker >= 0) sw_sched_fail_worker(sched_, worker, now_s());
    done_.fetch_add(1);
  }
  ::close(fd);
}

void MasterServer::stop() {
  if (listen_fd_ < 0 && !accept_thread_.joinable()) return;
  // wait until every slave reported DONE (they leave after their last completion)
  const double t0 = now_s();
  while (done_.load() < world_ && now_s() - t0 < 600.0) std::this_thread::sleep_for(std::chrono::milliseconds(1));
  if (listen_fd_ >= 0) { ::shutdown(listen_fd_, SHUT_RDWR); ::close(listen_fd_); listen_fd_ = -1; }
  if (accept_thread_.joinable()) accept_thread_.join();
  std::lock_guard<std::mutex> g(mu_);
  for (auto &t : conns_) if (t.joinable()) t.join();
  conns_.clear();
  if (sched_) {
    final_log_ = sw_sched_log_json(sched_);
    sw_sched_destroy(sched_);
    sched_ = nullptr;
  }
}

SchedClient::~SchedClient() {
  if (fd_ >= 0) ::close(fd_);
}

void SchedClient::connect(const char *host, int port, int rank, double timeout_s, uint64_t plan_hash) {
  rank_ = rank;
  const double t0 = now_s();
  addrinfo hints{}, *res = nullptr;
  hints.ai_family = AF_INET;
  hints.ai_socktype = SOCK_STREAM;
  if (getaddrinfo(host, std::to_string(port).c_str(), &hints, &res) != 0 || !res)
    throw Error(SW_ENET, std::string("slave: cannot resolve ") + host);
  while (true) {
    fd_ = ::socket(AF_INET, SOCK_STREAM, 0);
    if (fd_ >= 0 && ::connect(fd_, res->ai_addr, res->ai_addrlen) == 0) break;
    if (fd_ >= 0) ::close(fd_);
    fd_ = -1;
    if (now_s() - t0 > timeout_s) {
      freeaddrinfo(res);
      throw Error(SW_ENET, "slave: cannot reach the master at " + std::string(host) + ":" + std::to_string(port));
    }
    // retry quickly: every rank's GPU waits (and is timed) until all slaves registered
    std::this_thread::sleep_for(std::chrono::microseconds(500));
  }
  freeaddrinfo(res);
  nodelay(fd_);
  // "the slaves can register themselves in the master" (P16 §IV)
  if (call(kHello, 0, 0, 0, 0, 0, nullptr, plan_hash) < 0) {
    ::close(fd_);
    fd_ = -1;
    throw Error(SW_ENET, "slave: the master refused rank " + std::to_string(rank) +
                             ": its unit table differs from rank 0's (different inputs or options)");
  }
}

int32_t SchedClient::call(int32_t op, int32_t unit, int32_t cap, double t, double cells, double sec,
                          std::vector<int32_t> *extra, uint64_t hash) {
  Msg m{op, rank_, unit, cap, t, cells, sec, hash};
  RepHdr h;
  if (!send_all(fd_, &m, sizeof(m)) || !recv_all(fd_, &h, sizeof(h)))
    throw Error(SW_ENET, "slave: lost the connection to the master");
  std::vector<int32_t> tmp;
  std::vector<int32_t> &e = extra ? *extra : tmp;
  e.resize(h.nextra);
  if (h.nextra && !recv_all(fd_, e.data(), sizeof(int32_t) * h.nextra))
    throw Error(SW_ENET, "slave: lost the connection to the master");
  return h.rc;
}

int32_t SchedClient::request(double t, int32_t *out, int32_t cap) {
  std::vector<int32_t> e;
  const int32_t rc = call(kRequest, 0, cap, t, 0, 0, &e);
  for (int32_t k = 0; k < rc && k < (int32_t)e.size(); k++) out[k] = e[k];
  return rc;
}
int32_t SchedClient::request_wait(double t, int32_t *out, int32_t cap, double timeout_s) {
  std::vector<int32_t> e;
  const int32_t rc = call(kRequestWait, 0, cap, t, 0, timeout_s, &e);
  for (int32_t k = 0; k < rc && k < (int32_t)e.size(); k++) out[k] = e[k];
  return rc;
}
int64_t SchedClient::counter(int32_t which) {
  std::vector<int32_t> e;
  call(kCounters, 0, 0, 0, 0, 0, &e);
  if (e.size() < 3) return 0;
  return which == 0 ? e[0] : which == 1 ? e[1] : which == 3 ? e[2] : 0;
}
void SchedClient::report(double t, double cells, double sec) { call(kReport, 0, 0, t, cells, sec, nullptr); }
int32_t SchedClient::complete(int32_t unit, double t) { return call(kComplete, unit, 0, t, 0, 0, nullptr); }
void SchedClient::abandon(int32_t unit, double t) { call(kAbandon, unit, 0, t, 0, 0, nullptr); }
int32_t SchedClient::start(int32_t unit, double t) { return call(kStart, unit, 0, t, 0, 0, nullptr); }
int32_t SchedClient::is_finished(int32_t unit) {
  const double t = now_s();
  if (t - last_refresh_ > 5e-4 || unit / 32 >= (int32_t)finished_.size()) {
    const int32_t n = std::max<int32_t>(unit + 1, (int32_t)finished_.size() * 32);
    call(kFinishedMap, 0, n, t, 0, 0, &finished_);
    last_refresh_ = t;
  }
  if (unit / 32 >= (int32_t)finished_.size()) return 0;
  return (finished_[unit / 32] >> (unit % 32)) & 1;
}
void SchedClient::done() {
  std::vector<int32_t> e;
  call(kCounters, 0, 0, 0, 0, 0, &e);
  if (e.size() >= 3) { req_ = e[0]; wa_ = e[1]; grants_ = e[2]; }
  call(kDone, 0, 0, 0, 0, 0, nullptr);
  ::close(fd_);
  fd_ = -1;
}

}  // namespace sw

// ---- C-ABI wrappers (include/sw_sched.h) --------------------------------------------------
struct sw_master { sw::MasterServer s; };
struct sw_slave { sw::SchedClient c; };

namespace sw { void set_last_error(const std::string &m); }

extern "C" {

sw_master *sw_master_start(int32_t port, int32_t world, int32_t n_units, const int64_t *unit_cells,
                           int32_t policy, int32_t wa, int32_t omega, uint64_t plan_hash) {
  auto *m = new sw_master();
  try {
    m->s.start(port, world, n_units, unit_cells, policy, wa, omega, plan_hash);
    return m;
  } catch (const std::exception &e) {
    sw::set_last_error(e.what());
    delete m;
    return nullptr;
  }
}
void sw_master_stop(sw_master *m) {
  if (!m) return;
  m->s.stop();
  delete m;
}
sw_slave *sw_slave_connect(const char *host, int32_t port, int32_t rank, double timeout_s,
                           uint64_t plan_hash) {
  auto *c = new sw_slave();
  try {
    c->c.connect(host, port, rank, timeout_s, plan_hash);
    return c;
  } catch (const std::exception &e) {
    sw::set_last_error(e.what());
    delete c;
    return nullptr;
  }
}
static double clk() {
  using namespace std::chrono;
  return duration<double>(steady_clock::now().time_since_epoch()).count();
}
int32_t sw_slave_request(sw_slave *c, int32_t *out, int32_t cap) {
  try { return c->c.request(clk(), out, cap); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
int32_t sw_slave_request_wait(sw_slave *c, int32_t *out, int32_t cap, double timeout_s) {
  try { return c->c.request_wait(clk(), out, cap, timeout_s); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
int64_t sw_slave_counter(sw_slave *c, int32_t which) {
  try { return c->c.counter(which); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
void sw_slave_report(sw_slave *c, double cells, double seconds) {
  try { c->c.report(clk(), cells, seconds); } catch (const std::exception &e) { sw::set_last_error(e.what()); }
}
int32_t sw_slave_complete(sw_slave *c, int32_t unit) {
  try { return c->c.complete(unit, clk()); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
void sw_slave_abandon(sw_slave *c, int32_t unit) {
  try { c->c.abandon(unit, clk()); } catch (const std::exception &e) { sw::set_last_error(e.what()); }
}
int32_t sw_slave_start(sw_slave *c, int32_t unit) {
  try { return c->c.start(unit, clk()); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
int32_t sw_slave_is_finished(sw_slave *c, int32_t unit) {
  try { return c->c.is_finished(unit); } catch (const std::exception &e) { sw::set_last_error(e.what()); return -2; }
}
void sw_slave_done(sw_slave *c) {
  if (!c) return;
  try { c->c.done(); } catch (const std::exception &e) { sw::set_last_error(e.what()); }
  delete c;
}

}  // extern "C"
